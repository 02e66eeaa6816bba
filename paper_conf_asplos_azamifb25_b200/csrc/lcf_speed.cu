// lcf_speed.cu — SPspeed / DPspeed (§3.1) on sm_100a.
//
// One 256-thread CTA per 16 KiB chunk (L104), chunk index from a ticket so the
// decoupled look-back (L122) only waits on CTAs that already run. Warp w owns
// subchunks 4w..4w+3 (512 B each, L118): one coalesced 16-byte load per lane
// per subchunk, so a lane holds K = 4 (f32) or 2 (f64) consecutive words.
//
// Encode: DIFFMS in registers (neighbour word by shuffle) → per-subchunk width
// by a warp max-reduction of bit lengths → TCMS retry if the maximum has no
// leading zero (L114) → the chunk size is known before any packing, so the
// aggregate is published at once → lanes emit their K·w-bit strings into the
// shared-memory output buffer (lcf::emit_bits_warp) while warp 0 resolves the
// look-back → coalesced 16-byte stores at the resolved offset.
// Decode: the size-table entry gives the aggregate immediately → look-back →
// 16-byte loads of the payload into shared memory → each lane funnel-shifts
// its K fields out → unTCMS → DIFFMS⁻¹ as a block-wide prefix sum (L132).
#include "lcf_kernels.cuh"

namespace lcf {

namespace {

constexpr int kThreads = 256, kWarps = 8, kSubPerWarp = 4;

template <typename U> struct Cfg {
  static constexpr int W = 8 * sizeof(U);
  static constexpr int CW = 16384 / sizeof(U);  // chunk words
  static constexpr int SW = 512 / sizeof(U);    // subchunk words (L118)
  static constexpr int K = SW / 32;             // words per lane per subchunk
};

// K consecutive words of one lane <-> one 16-byte vector
template <typename U> __device__ __forceinline__ void unpack16(const uint4& q, U* v);
template <> __device__ __forceinline__ void unpack16<uint32_t>(const uint4& q, uint32_t* v) {
  v[0] = q.x; v[1] = q.y; v[2] = q.z; v[3] = q.w;
}
template <> __device__ __forceinline__ void unpack16<uint64_t>(const uint4& q, uint64_t* v) {
  v[0] = ((uint64_t)q.y << 32) | q.x;
  v[1] = ((uint64_t)q.w << 32) | q.z;
}
template <typename U> __device__ __forceinline__ uint4 pack16(const U* v);
template <> __device__ __forceinline__ uint4 pack16<uint32_t>(const uint32_t* v) {
  return make_uint4(v[0], v[1], v[2], v[3]);
}
template <> __device__ __forceinline__ uint4 pack16<uint64_t>(const uint64_t* v) {
  return make_uint4((uint32_t)v[0], (uint32_t)(v[0] >> 32), (uint32_t)v[1], (uint32_t)(v[1] >> 32));
}

// Lane string of K fields of width w (K·w ≤ 128 bits) as a 128-bit value.
__device__ __forceinline__ void make_string(const uint32_t* v, unsigned w, uint64_t& lo, uint64_t& hi) {
  const uint64_t a = (uint64_t)v[0] | ((uint64_t)v[1] << w);  // 2w bits
  const uint64_t b = (uint64_t)v[2] | ((uint64_t)v[3] << w);
  const unsigned s = 2 * w;
  if (s == 64) { lo = a; hi = b; }
  else if (s == 0) { lo = 0; hi = 0; }
  else { lo = a | (b << s); hi = b >> (64 - s); }
}
__device__ __forceinline__ void make_string(const uint64_t* v, unsigned w, uint64_t& lo, uint64_t& hi) {
  if (w == 64) { lo = v[0]; hi = v[1]; }
  else if (w == 0) { lo = 0; hi = 0; }
  else { lo = v[0] | (v[1] << w); hi = v[1] >> (64 - w); }
}
__device__ __forceinline__ void split_string(uint64_t lo, uint64_t hi, unsigned w, uint32_t* v) {
  const uint32_t m = w >= 32 ? 0xFFFFFFFFu : ((1u << w) - 1u);
  v[0] = (uint32_t)lo & m;
  v[1] = (uint32_t)(w >= 64 ? 0 : (lo >> w)) & m;
  uint64_t l2 = lo, h2 = hi;
  shr128(l2, h2, 2 * w);
  v[2] = (uint32_t)l2 & m;
  v[3] = (uint32_t)(w >= 64 ? 0 : (l2 >> w)) & m;
  if (w == 0) v[0] = v[1] = v[2] = v[3] = 0;
}
__device__ __forceinline__ void split_string(uint64_t lo, uint64_t hi, unsigned w, uint64_t* v) {
  const uint64_t m = mask64(w);
  v[0] = lo & m;
  uint64_t l2 = lo, h2 = hi;
  shr128(l2, h2, w);
  v[1] = l2 & m;
  if (w == 0) v[0] = v[1] = 0;
}

template <typename U> __device__ __forceinline__ U shfl_up1(U v) { return __shfl_up_sync(0xFFFFFFFFu, v, 1); }
template <typename U> __device__ __forceinline__ U shfl_idx(U v, int l) { return __shfl_sync(0xFFFFFFFFu, v, l); }

template <typename U>
__global__ void __launch_bounds__(kThreads) speed_encode_kernel(EncArgs a, LaunchCtx ctx) {
  using C = Cfg<U>;
  constexpr int W = C::W, CW = C::CW, SW = C::SW, K = C::K;
  __shared__ __align__(16) uint32_t s_out[(kChunkBytes + 64) / 4];
  __shared__ uint32_t s_subbytes[32], s_suboff[32];
  __shared__ uint64_t s_c, s_excl;
  __shared__ uint32_t s_len, s_raw;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) s_c = atomicAdd(ctx.ticket, 1ull) - ctx.ticket_base;
  __syncthreads();
  const uint64_t c = s_c;
  const uint64_t gc = a.first_chunk + c;
  const uint32_t m = (uint32_t)umin64((uint64_t)CW, a.n_words_total - gc * CW);
  const U* src = reinterpret_cast<const U*>(a.in) + c * CW;

  // ---- load (16 B per lane per subchunk) and DIFFMS (L110–112) ----
  U v[kSubPerWarp][K];
#pragma unroll
  for (int q = 0; q < kSubPerWarp; ++q) {
    const uint32_t i0 = (warp * kSubPerWarp + q) * SW + lane * K;
    if (i0 + K <= m) {
      unpack16<U>(__ldcs(reinterpret_cast<const uint4*>(src + i0)), v[q]);
    } else {
#pragma unroll
      for (int j = 0; j < K; ++j) v[q][j] = (i0 + j < m) ? src[i0 + j] : (U)0;
    }
  }
  const uint32_t wfirst = warp * kSubPerWarp * SW;
  U carry = (warp > 0 && wfirst - 1 < m) ? src[wfirst - 1] : (U)0;
  uint32_t wq[kSubPerWarp];
#pragma unroll
  for (int q = 0; q < kSubPerWarp; ++q) {
    const U next_carry = shfl_idx(v[q][K - 1], 31);
    U p = shfl_up1(v[q][K - 1]);
    if (lane == 0) p = carry;
    carry = next_carry;
    const uint32_t i0 = (warp * kSubPerWarp + q) * SW + lane * K;
#pragma unroll
    for (int j = K - 1; j >= 0; --j) {
      const U prev = j ? v[q][j - 1] : p;
      v[q][j] = (i0 + j < m) ? tcms((U)(v[q][j] - prev)) : (U)0;
    }
    // ---- MPLG width per subchunk (L114–118) ----
    int bl = 0;
#pragma unroll
    for (int j = 0; j < K; ++j) bl = max(bl, bitlen(v[q][j]));
    int wmax = (int)__reduce_max_sync(0xFFFFFFFFu, (unsigned)bl);
    uint32_t flag = 0;
    if (wmax == W) {  // maximum has no leading zero: TCMS once more
      flag = 1;
      bl = 0;
#pragma unroll
      for (int j = 0; j < K; ++j) {
        v[q][j] = tcms(v[q][j]);
        bl = max(bl, bitlen(v[q][j]));
      }
      wmax = (int)__reduce_max_sync(0xFFFFFFFFu, (unsigned)bl);
    }
    wq[q] = (uint32_t)wmax | (flag << 7);
    if (lane == 0) {
      const int s = warp * kSubPerWarp + q;
      const int64_t rem = (int64_t)m - (int64_t)s * SW;
      const uint32_t ms = rem <= 0 ? 0u : (uint32_t)(rem < SW ? rem : SW);
      s_subbytes[s] = (ms * (uint32_t)wmax + 7) / 8;
      reinterpret_cast<uint8_t*>(s_out)[s] = ms ? (uint8_t)wq[q] : (uint8_t)0;
    }
  }
  __syncthreads();

  // ---- chunk size, raw decision, aggregate published before packing ----
  if (warp == 0) {
    const uint32_t S = (m + SW - 1) / SW;
    const uint32_t hdr = (S + 7) & ~7u;
    const uint32_t b = s_subbytes[lane];
    uint32_t incl = b;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(0xFFFFFFFFu, incl, d);
      if (lane >= d) incl += o;
    }
    s_suboff[lane] = hdr + incl - b;
    const uint32_t total = hdr + __shfl_sync(0xFFFFFFFFu, incl, 31);
    const uint32_t raw_len = m * (uint32_t)sizeof(U);
    const bool raw = total >= raw_len;  // L104, ties → raw
    const uint32_t len = raw ? raw_len : total;
    if (lane == 0) {
      s_len = len;
      s_raw = raw;
      lookback_publish(ctx, c, round16(len));
    }
    if (!raw && lane < 16 && len + lane < round16(len))  // zero pad bytes
      reinterpret_cast<uint8_t*>(s_out)[len + lane] = 0;
  }
  __syncthreads();
  const uint32_t len = s_len;
  const bool raw = s_raw;

  if (warp == 0) {
    const uint64_t excl = lookback_warp(ctx, c, round16(len));
    if (lane == 0) s_excl = excl;
  }
  if (!raw) {
#pragma unroll
    for (int q = 0; q < kSubPerWarp; ++q) {
      const uint32_t w = wq[q] & 0x7F;
      if (w == 0) continue;
      const int s = warp * kSubPerWarp + q;
      const unsigned Lb = K * w;
      uint64_t lo, hi;
      make_string(v[q], w, lo, hi);
      emit_bits_warp(s_out, (uint64_t)s_suboff[s] * 8 + (uint64_t)lane * Lb, Lb, lo, hi, false, Lb >= 32);
    }
  }
  __syncthreads();

  // ---- store at the resolved offset (16-byte granules) ----
  uint8_t* dst = a.payload + s_excl;
  const uint32_t n16 = (uint32_t)(round16(len) / 16);
  if (!raw) {
    for (uint32_t i = tid; i < n16; i += kThreads)
      __stcs(reinterpret_cast<uint4*>(dst) + i, reinterpret_cast<const uint4*>(s_out)[i]);
  } else {
    const uint8_t* rsrc = reinterpret_cast<const uint8_t*>(src);
    for (uint32_t i = tid; i < n16; i += kThreads) {
      uint4 val;
      if (16 * i + 16 <= len) {
        val = __ldcs(reinterpret_cast<const uint4*>(rsrc) + i);
      } else {
        uint32_t wv[4];
#pragma unroll
        for (int j = 0; j < 4; ++j)
          wv[j] = (16 * i + 4 * j < len) ? reinterpret_cast<const uint32_t*>(rsrc)[4 * i + j] : 0u;
        val = make_uint4(wv[0], wv[1], wv[2], wv[3]);
      }
      __stcs(reinterpret_cast<uint4*>(dst) + i, val);
    }
  }
  if (tid == 0) {
    a.table[c] = len | (raw ? kRawFlag : 0u);
    if (c == a.n_chunks - 1) finish_encode(a, s_excl + round16(len));
  }
  if (c == 0 && tid < 16 && tid < a.pad_len) a.pad_start[tid] = 0;
}

template <typename U>
__global__ void __launch_bounds__(kThreads) speed_decode_kernel(DecArgs a, LaunchCtx ctx) {
  using C = Cfg<U>;
  constexpr int W = C::W, CW = C::CW, SW = C::SW, K = C::K;
  __shared__ __align__(16) uint32_t s_in[(kChunkBytes + 64) / 4];
  __shared__ uint32_t s_suboff[32], s_hdr[32];
  __shared__ U s_wtot[kWarps];
  __shared__ uint64_t s_excl;
  __shared__ DecChunk s_ch;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) s_ch = decode_chunk_begin(a, ctx, sizeof(U), CW);
  __syncthreads();
  const DecChunk ch = s_ch;
  if (!ch.ok) return;
  if (warp == 0) {
    const uint64_t excl = lookback_warp(ctx, ch.c, round16(ch.len));
    if (lane == 0) {
      s_excl = excl;
      const uint64_t end = excl + round16(ch.len);
      if (end > ch.payload_bytes || (ch.c == ch.n_chunks - 1 && end != ch.payload_bytes)) {
        record_error(ctx, DERR_CORRUPT);
        s_ch.ok = 0;
      }
    }
  }
  __syncthreads();
  if (!s_ch.ok) return;
  const uint8_t* psrc = a.stream + ch.base + s_excl;
  const uint32_t n16 = (uint32_t)(round16(ch.len) / 16);
  U* dst = reinterpret_cast<U*>(a.out) + ch.c * CW;
  const uint32_t m = ch.m;

  if (ch.raw) {  // raw chunk: copy (len = m·sizeof(U))
    for (uint32_t i = tid; i < n16; i += kThreads) {
      const uint4 val = __ldcs(reinterpret_cast<const uint4*>(psrc) + i);
      if (16 * i + 16 <= ch.len) {
        __stcs(reinterpret_cast<uint4*>(dst) + i, val);
      } else {
        const uint32_t wv[4] = {val.x, val.y, val.z, val.w};
        for (int j = 0; j < 4; ++j)
          if (16 * i + 4 * j < ch.len) reinterpret_cast<uint32_t*>(dst)[4 * i + j] = wv[j];
      }
    }
    return;
  }
  for (uint32_t i = tid; i < n16; i += kThreads)
    reinterpret_cast<uint4*>(s_in)[i] = __ldcs(reinterpret_cast<const uint4*>(psrc) + i);
  __syncthreads();

  // ---- MPLG header: widths, flags, subchunk offsets (L114–118) ----
  if (warp == 0) {
    const uint32_t S = (m + SW - 1) / SW;
    const uint32_t hdr = (S + 7) & ~7u;
    const int64_t rem = (int64_t)m - (int64_t)lane * SW;
    const uint32_t ms = rem <= 0 ? 0u : (uint32_t)(rem < SW ? rem : SW);
    uint32_t h = ms ? reinterpret_cast<const uint8_t*>(s_in)[lane] : 0u;
    bool bad = (h & 0x7F) > (uint32_t)W;
    if (bad) h = 0;
    const uint32_t b = (ms * (h & 0x7F) + 7) / 8;
    uint32_t incl = b;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(0xFFFFFFFFu, incl, d);
      if (lane >= d) incl += o;
    }
    s_suboff[lane] = hdr + incl - b;
    s_hdr[lane] = h;
    const uint32_t total = hdr + __shfl_sync(0xFFFFFFFFu, incl, 31);
    if (__any_sync(0xFFFFFFFFu, bad) || total != ch.len || hdr > ch.len) {
      if (lane == 0) {
        record_error(ctx, DERR_CORRUPT);
        s_ch.ok = 0;
      }
    }
  }
  __syncthreads();
  if (!s_ch.ok) return;

  // ---- unpack K fields per lane, unTCMS, local sums ----
  const uint32_t nwords = n16 * 4;
  U d[kSubPerWarp][K];
  U lane_tot[kSubPerWarp];
#pragma unroll
  for (int q = 0; q < kSubPerWarp; ++q) {
    const int s = warp * kSubPerWarp + q;
    const uint32_t h = s_hdr[s];
    const uint32_t w = h & 0x7F;
    const uint64_t off = (uint64_t)s_suboff[s] * 8 + (uint64_t)lane * K * w;
    const uint32_t F = (uint32_t)(off >> 5), r = (uint32_t)(off & 31);
    uint32_t t[5];
#pragma unroll
    for (int j = 0; j < 5; ++j) t[j] = (w && F + j < nwords) ? s_in[F + j] : 0u;
    const uint64_t lo = (uint64_t)__funnelshift_r(t[0], t[1], r) | ((uint64_t)__funnelshift_r(t[1], t[2], r) << 32);
    const uint64_t hi = (uint64_t)__funnelshift_r(t[2], t[3], r) | ((uint64_t)__funnelshift_r(t[3], t[4], r) << 32);
    split_string(lo, hi, w, d[q]);
    U tot = 0;
#pragma unroll
    for (int j = 0; j < K; ++j) {
      U u = d[q][j];
      if (h >> 7) u = tcms_inv(u);
      d[q][j] = tcms_inv(u);  // DIFFMS difference
      tot += d[q][j];
    }
    lane_tot[q] = tot;
  }
  // ---- DIFFMS⁻¹: block-wide inclusive prefix sum mod 2^W (L132) ----
  U wcarry = 0;
  U excl_q[kSubPerWarp];
#pragma unroll
  for (int q = 0; q < kSubPerWarp; ++q) {
    U incl = lane_tot[q];
#pragma unroll
    for (int dd = 1; dd < 32; dd <<= 1) {
      const U o = __shfl_up_sync(0xFFFFFFFFu, incl, dd);
      if (lane >= dd) incl += o;
    }
    excl_q[q] = wcarry + incl - lane_tot[q];
    wcarry += shfl_idx(incl, 31);
  }
  if (lane == 0) s_wtot[warp] = wcarry;
  __syncthreads();
  U wbase = 0;
  for (int i = 0; i < warp; ++i) wbase += s_wtot[i];
#pragma unroll
  for (int q = 0; q < kSubPerWarp; ++q) {
    U run = wbase + excl_q[q];
    U x[K];
#pragma unroll
    for (int j = 0; j < K; ++j) {
      run += d[q][j];
      x[j] = run;
    }
    const uint32_t i0 = (warp * kSubPerWarp + q) * SW + lane * K;
    if (i0 + K <= m) {
      __stcs(reinterpret_cast<uint4*>(dst + i0), pack16<U>(x));
    } else {
#pragma unroll
      for (int j = 0; j < K; ++j)
        if (i0 + j < m) dst[i0 + j] = x[j];
    }
  }
}

}  // namespace

template <typename U> void launch_speed_encode(const EncArgs& a, const LaunchCtx& ctx, cudaStream_t st) {
  speed_encode_kernel<U><<<(unsigned)a.n_chunks, kThreads, 0, st>>>(a, ctx);
}
template <typename U> void launch_speed_decode(const DecArgs& a, const LaunchCtx& ctx, unsigned grid, cudaStream_t st) {
  speed_decode_kernel<U><<<grid, kThreads, 0, st>>>(a, ctx);
}
template void launch_speed_encode<uint32_t>(const EncArgs&, const LaunchCtx&, cudaStream_t);
template void launch_speed_encode<uint64_t>(const EncArgs&, const LaunchCtx&, cudaStream_t);
template void launch_speed_decode<uint32_t>(const DecArgs&, const LaunchCtx&, unsigned, cudaStream_t);
template void launch_speed_decode<uint64_t>(const DecArgs&, const LaunchCtx&, unsigned, cudaStream_t);

}  // namespace lcf
