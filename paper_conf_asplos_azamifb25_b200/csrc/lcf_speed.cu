// lcf_speed.cu — SPspeed / DPspeed (§3.1) on sm_100a.
//
// Persistent, warp-specialised CTAs; chunks (16 KiB, L104) are handed out by a
// global ticket so the decoupled look-back (L122) only ever waits on chunks
// that running CTAs already own.
//
// Encode CTA (320 threads):
//   warp 0  loader : ticket → 1-D TMA bulk load of the chunk into a
//                    shared-memory stage (1 stage: it is released as soon as
//                    the compute warps hold the chunk in registers; mbarrier
//                    complete_tx)
//   warp 1  storer : decoupled look-back for the chunk's output offset →
//                    1-D TMA bulk store of the packed chunk → size-table entry
//   warps 2-9      : DIFFMS in registers (L110–112) → per-subchunk width by a
//                    warp OR-reduction (bitlen(max) = bitlen(OR)) with the TCMS
//                    retry (L114) → aggregate published as soon as the size is
//                    known → bit packing (L116) into a 2-slot output ring.
// Decode CTA (288 threads):
//   warp 0  loader : ticket → size entry → aggregate published at once →
//                    look-back → TMA bulk load of the payload (3 stages)
//   warps 1-8      : unpack (funnel shifts) → unTCMS → DIFFMS⁻¹ as a CTA-wide
//                    prefix sum (L132) → 16-byte coalesced stores.
// Each compute warp owns subchunks 4w..4w+3 (512 B, L118); a lane holds K = 4
// (f32) or 2 (f64) consecutive words of each.
#include "lcf_persist.cuh"

namespace lcf {

namespace {

constexpr int kCompWarps = 8, kSubPerWarp = 4;
// Encoder buffering (measured on B200, NYX / Miranda / CESM): the input stage
// is released as soon as the compute warps hold the chunk in registers, so one
// input stage suffices, and a third output slot absorbs the storer's look-back
// waits (2→1 input stages, 2→3 output slots: −4…8 % compress time). Round 2:
// 2 output slots with a 48-register bound fit 4 CTAs/SM (3 slots at 62
// registers: 3 CTAs/SM): NYX velocity 229 → 225 µs, HACC xx 426 → 421 µs,
// Miranda density 130 → 129 µs, CESM T 23.3 → 24.6 µs.
#ifndef LCF_ENC_STAGES
#define LCF_ENC_STAGES 1
#endif
#ifndef LCF_ENC_OUT
#define LCF_ENC_OUT 2
#endif
#ifndef LCF_ENC_MINB
#define LCF_ENC_MINB 4
#endif
#ifndef LCF_ENC_STORERS
#define LCF_ENC_STORERS 1
#endif
#ifndef LCF_DEC_STAGES
#define LCF_DEC_STAGES 3
#endif
#ifndef LCF_DEC_BATCH
#define LCF_DEC_BATCH 4
#endif
constexpr int kEncStages = LCF_ENC_STAGES, kEncOut = LCF_ENC_OUT, kStorers = LCF_ENC_STORERS;
constexpr int kDecStages = LCF_DEC_STAGES, kDecBatch = LCF_DEC_BATCH;
static_assert(kStorers == 1 || kEncOut % kStorers == 0, "each output slot belongs to one storer");
constexpr int kEncThreads = (1 + kStorers + kCompWarps) * 32;
constexpr int kDecThreads = (1 + kCompWarps) * 32;
constexpr uint32_t kCompThreads = kCompWarps * 32;
constexpr uint32_t kBarCompute = 1;  // named barrier of the compute warps

template <typename U> struct Cfg {
  static constexpr int W = 8 * sizeof(U);
  static constexpr int CW = 16384 / sizeof(U);  // chunk words
  static constexpr int SW = 512 / sizeof(U);    // subchunk words (L118)
  static constexpr int K = SW / 32;             // words per lane per subchunk
};

struct EncSmem {
  alignas(128) uint32_t in[kEncStages][kChunkBytes / 4];
  alignas(128) uint32_t out[kEncOut][(kChunkBytes + 64) / 4];
  uint64_t full_in[kEncStages], empty_in[kEncStages], full_out[kEncOut], empty_out[kEncOut];
  uint64_t in_chunk[kEncStages], out_chunk[kEncOut];
  uint32_t out_len[kEncOut], out_raw[kEncOut];
  uint32_t hdr[2][32];
};

// Decoder payload stages per word type: the f32 decoder at 40 registers fits 5
// CTAs per SM with 2 stages (NYX velocity 184 → 182 µs, HACC xx 341 → 334 µs);
// the f64 decoder measured slower that way (123 → 124.5 µs) and keeps 3 stages
// at 4 CTAs per SM.
#ifndef LCF_DEC_STAGES_U32
#define LCF_DEC_STAGES_U32 2
#endif
template <typename U> struct DecCfg {
  static constexpr int kStages = sizeof(U) == 4 ? LCF_DEC_STAGES_U32 : kDecStages;
  static constexpr int kMinBlocks = sizeof(U) == 4 && LCF_DEC_STAGES_U32 == 2 ? 5 : 4;
};
template <typename U> struct DecSmem {
  static constexpr int kDecStages = DecCfg<U>::kStages;
  alignas(128) uint32_t in[kDecStages][(kChunkBytes + 64) / 4];
  uint64_t full_in[kDecStages], empty_in[kDecStages];
  uint64_t chunk[kDecStages];
  uint32_t len[kDecStages], flags[kDecStages];  // flags: bit0 raw, bit1 bad
  U wtot[2][kCompWarps];
};

// ---- word <-> 16-byte vector --------------------------------------------------
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

// ---- MPLG width: bitlen(max) == bitlen(OR) over the subchunk --------------------
// LCF_REDUX: 0 = __reduce_or_sync, 1 = redux.sync in inline PTX, 2 = a
// butterfly of shuffles
#ifndef LCF_REDUX
#define LCF_REDUX 0
#endif
__device__ __forceinline__ uint32_t warp_or(uint32_t x) {
#if LCF_REDUX == 1
  uint32_t o;
  asm volatile("redux.sync.or.b32 %0, %1, 0xffffffff;" : "=r"(o) : "r"(x));
  return o;
#elif LCF_REDUX == 2
#pragma unroll
  for (int d = 16; d >= 1; d >>= 1) x |= __shfl_xor_sync(0xFFFFFFFFu, x, d);
  return x;
#else
  return __reduce_or_sync(0xFFFFFFFFu, x);
#endif
}
__device__ __forceinline__ uint32_t warp_width(const uint32_t* v) {
  const uint32_t o = warp_or(v[0] | v[1] | v[2] | v[3]);
  return 32 - __clz(o);
}
__device__ __forceinline__ uint32_t warp_width(const uint64_t* v) {
  const uint64_t x = v[0] | v[1];
  const uint32_t hi = warp_or((uint32_t)(x >> 32));
  const uint32_t lo = warp_or((uint32_t)x);
  return hi ? 64 - __clz(hi) : 32 - __clz(lo);
}

// ---- a lane's K fields of width w as one bit string (4 words, ≤ 128 bits) -------
__device__ __forceinline__ void make_string(const uint32_t* v, uint32_t w, uint32_t* S) {
  const uint32_t a_lo = v[0] | shl_c(v[1], w), a_hi = __funnelshift_lc(v[1], 0u, w);
  const uint32_t b_lo = v[2] | shl_c(v[3], w), b_hi = __funnelshift_lc(v[3], 0u, w);
  if (w >= 16) {  // b goes to bit 2w ≥ 32
    const uint32_t t = 2 * w - 32;
    S[0] = a_lo;
    S[1] = a_hi | shl_c(b_lo, t);
    S[2] = __funnelshift_lc(b_lo, b_hi, t);
    S[3] = __funnelshift_lc(b_hi, 0u, t);
  } else {
    const uint32_t t = 2 * w;
    S[0] = a_lo | shl_c(b_lo, t);
    S[1] = a_hi | __funnelshift_lc(b_lo, b_hi, t);
    S[2] = __funnelshift_lc(b_hi, 0u, t);
    S[3] = 0;
  }
}
__device__ __forceinline__ void make_string(const uint64_t* v, uint32_t w, uint32_t* S) {
  const uint32_t a0 = (uint32_t)v[0], a1 = (uint32_t)(v[0] >> 32), b0 = (uint32_t)v[1], b1 = (uint32_t)(v[1] >> 32);
  if (w >= 32) {  // v1 goes to bit w = 32 + s
    const uint32_t s = w - 32;
    S[0] = a0;
    S[1] = a1 | shl_c(b0, s);
    S[2] = __funnelshift_lc(b0, b1, s);
    S[3] = __funnelshift_lc(b1, 0u, s);
  } else {
    S[0] = a0 | shl_c(b0, w);
    S[1] = a1 | __funnelshift_lc(b0, b1, w);
    S[2] = __funnelshift_lc(b1, 0u, w);
    S[3] = 0;
  }
}

// Lanes' strings of equal length L = K·w ≥ 32 bits, lane l at bit l·L of the
// word-aligned subchunk stream `buf`: every word is shared by ≤ 2 lanes, so one
// shuffle hands the partial last word to the next lane. Every word of the
// stream is written exactly once.
__device__ __forceinline__ void emit_equal(uint32_t* buf, uint32_t lane, uint32_t L, const uint32_t* S) {
  const uint32_t P = lane * L, F = P >> 5, r = P & 31;
  uint32_t T[5];
  T[0] = S[0] << r;
  T[1] = __funnelshift_l(S[0], S[1], r);
  T[2] = __funnelshift_l(S[1], S[2], r);
  T[3] = __funnelshift_l(S[2], S[3], r);
  T[4] = __funnelshift_l(S[3], 0u, r);
  const uint32_t e = (r + L - 1) >> 5;  // index of the last word touched (0..4)
  const uint32_t last = e == 1 ? T[1] : e == 2 ? T[2] : e == 3 ? T[3] : e == 4 ? T[4] : T[0];
  const uint32_t in = __shfl_up_sync(0xFFFFFFFFu, last, 1);
  if (r) T[0] |= in;
  const bool keep_last = ((r + L) & 31) == 0 || lane == 31;
#pragma unroll
  for (uint32_t j = 0; j < 5; ++j)
    if (j < e || (j == e && keep_last)) buf[F + j] = T[j];
}

// LCF_ENC_OR: the same strings OR-ed into an output slot that is zero by
// invariant (the storer re-zeroes what it stored before handing the slot back;
// zeroing by the compute warps behind one more barrier measured equal, a third
// output slot at 3 CTAs/SM slower):
// no shuffle of the partial word, no select of the last word, one predicated
// shared reduction per touched word.
#ifndef LCF_ENC_OR
#define LCF_ENC_OR 1
#endif
#ifndef LCF_ENC_OR_UNIFORM
#define LCF_ENC_OR_UNIFORM 1
#endif
__device__ __forceinline__ void emit_or(uint32_t* buf, uint32_t lane, uint32_t L, const uint32_t* S) {
  const uint32_t P = lane * L, F = P >> 5, r = P & 31;
  const uint32_t e = (r + L - 1) >> 5;  // index of the last word touched (0..4)
#if LCF_ENC_OR_UNIFORM
  // words past emax = (L + 30) / 32 (warp-uniform: L is the subchunk's) are
  // touched by no lane: uniform branches skip their shifts and reductions
  const uint32_t emax = (L + 30) >> 5;
  atomicOr(buf + F, S[0] << r);
  if (emax >= 1) {
    if (e >= 1) atomicOr(buf + F + 1, __funnelshift_l(S[0], S[1], r));
    if (emax >= 2) {
      if (e >= 2) atomicOr(buf + F + 2, __funnelshift_l(S[1], S[2], r));
      if (emax >= 3) {
        if (e >= 3) atomicOr(buf + F + 3, __funnelshift_l(S[2], S[3], r));
        if (emax >= 4 && e >= 4) atomicOr(buf + F + 4, __funnelshift_l(S[3], 0u, r));
      }
    }
  }
#else
  const uint32_t T[5] = {S[0] << r, __funnelshift_l(S[0], S[1], r), __funnelshift_l(S[1], S[2], r),
                         __funnelshift_l(S[2], S[3], r), __funnelshift_l(S[3], 0u, r)};
#pragma unroll
  for (uint32_t j = 0; j < 5; ++j)
    if (j <= e) atomicOr(buf + F + j, T[j]);
#endif
}

// ---- shared-memory field extraction (decode) ------------------------------------
__device__ __forceinline__ void split_string(const uint32_t* U4, uint32_t w, uint32_t* v) {
  const uint32_t m = w >= 32 ? 0xFFFFFFFFu : ((1u << w) - 1u);
  v[0] = U4[0] & m;
  v[1] = __funnelshift_rc(U4[0], U4[1], w) & m;
  uint32_t lo, hi, s;
  if (w >= 16) { lo = U4[1]; hi = U4[2]; s = 2 * w - 32; }
  else { lo = U4[0]; hi = U4[1]; s = 2 * w; }
  v[2] = __funnelshift_rc(lo, hi, s) & m;
  const uint32_t p3 = 3 * w, i3 = p3 >> 5, s3 = p3 & 31;
  const uint32_t x0 = i3 == 0 ? U4[0] : i3 == 1 ? U4[1] : i3 == 2 ? U4[2] : U4[3];
  const uint32_t x1 = i3 == 0 ? U4[1] : i3 == 1 ? U4[2] : U4[3];
  v[3] = __funnelshift_r(x0, x1, s3) & m;
}
__device__ __forceinline__ void split_string(const uint32_t* U4, uint32_t w, uint64_t* v) {
  // 32-bit pieces: field 0 = bits [0, w), field 1 = bits [w, 2w) of the window
  const uint32_t mlo = w >= 32 ? 0xFFFFFFFFu : ((1u << w) - 1u);
  const uint32_t mhi = w >= 64 ? 0xFFFFFFFFu : (w <= 32 ? 0u : ((1u << (w - 32)) - 1u));
  v[0] = ((uint64_t)(U4[1] & mhi) << 32) | (U4[0] & mlo);
  const uint32_t sh = w & 31;
  uint32_t a0, a1, a2;
  if (w >= 64) { a0 = U4[2]; a1 = U4[3]; a2 = 0; }
  else if (w >= 32) { a0 = U4[1]; a1 = U4[2]; a2 = U4[3]; }
  else { a0 = U4[0]; a1 = U4[1]; a2 = U4[2]; }
  const uint32_t lo = __funnelshift_r(a0, a1, sh) & mlo, hi = __funnelshift_r(a1, a2, sh) & mhi;
  v[1] = ((uint64_t)hi << 32) | lo;
}

// TCMS⁻¹ with −(u & 1) as one sign extension of bit 0 (bfe.s32 → SASS SGXT):
// 3 instructions per 32-bit word instead of 4. The decoder is ALU-pipe bound
// (SPspeed decode NYX velocity 192.5 → 190.5 µs, HACC xx 357 → 354 µs); the
// SPratio decoder measured 1.5 % slower with it, so it keeps tcms_inv.
__device__ __forceinline__ uint32_t sign_of_bit0(uint32_t u) {
  int32_t m;
  asm("bfe.s32 %0, %1, 0, 1;" : "=r"(m) : "r"((int32_t)u));
  return (uint32_t)m;
}
__device__ __forceinline__ uint32_t tcms_inv_sx(uint32_t u) { return (u >> 1) ^ sign_of_bit0(u); }
__device__ __forceinline__ uint64_t tcms_inv_sx(uint64_t u) {  // on 32-bit halves: one shared sign mask
  const uint32_t lo = (uint32_t)u, hi = (uint32_t)(u >> 32);
  const uint32_t m = sign_of_bit0(lo);
  return ((uint64_t)((hi >> 1) ^ m) << 32) | (__funnelshift_r(lo, hi, 1) ^ m);
}

template <typename U> __device__ __forceinline__ U shfl_up1(U v) { return __shfl_up_sync(0xFFFFFFFFu, v, 1); }
template <typename U> __device__ __forceinline__ U shfl_idx(U v, int l) { return __shfl_sync(0xFFFFFFFFu, v, l); }

// =================================== encode ======================================
template <typename U>
__device__ __forceinline__ void enc_compute(EncSmem& S, const EncArgs& a, const LaunchCtx& ctx, uint32_t cw,
                                            uint32_t lane) {
  using C = Cfg<U>;
  constexpr int W = C::W, CW = C::CW, SW = C::SW, K = C::K;
  for (uint32_t it = 0;; ++it) {
    const uint32_t s = it % kEncStages, ph = (it / kEncStages) & 1;
    const uint32_t o = it % kEncOut, pho = (it / kEncOut) & 1;
    mbar_wait(&S.full_in[s], ph);
    const uint64_t t = S.in_chunk[s];
    if (t == kNoChunk) {
      enc_forward_end<kEncOut, kStorers>(S, it, cw, lane);
      return;
    }
    if (cw == 0 && lane == 0) trace_stamp(a, t, 1);
    const uint32_t m = chunk_words(a.n_words_total, a.first_chunk + t, CW);
    const bool full = m == (uint32_t)CW;
    const U* in = reinterpret_cast<const U*>(S.in[s]);
    U v[kSubPerWarp][K];
#pragma unroll
    for (int q = 0; q < kSubPerWarp; ++q)
      unpack16<U>(reinterpret_cast<const uint4*>(in)[(cw * kSubPerWarp + q) * 32 + lane], v[q]);
    const uint32_t wfirst = cw * kSubPerWarp * SW;
    U carry = (cw > 0 && wfirst - 1 < m) ? in[wfirst - 1] : (U)0;
    __syncwarp();
    if (lane == 0) mbar_arrive(&S.empty_in[s]);  // stage consumed (raw chunks re-read global)

    // DIFFMS (L110–112) and MPLG widths with the TCMS retry (L114–118)
    uint32_t wq[kSubPerWarp];
#pragma unroll
    for (int q = 0; q < kSubPerWarp; ++q) {
      const U next_carry = shfl_idx(v[q][K - 1], 31);
      U p = shfl_up1(v[q][K - 1]);
      if (lane == 0) p = carry;
      carry = next_carry;
      const uint32_t i0 = (cw * kSubPerWarp + q) * SW + lane * K;
      if (full) {
#pragma unroll
        for (int j = K - 1; j >= 0; --j) v[q][j] = tcms((U)(v[q][j] - (j ? v[q][j - 1] : p)));
      } else {
#pragma unroll
        for (int j = K - 1; j >= 0; --j) {
          const U u = tcms((U)(v[q][j] - (j ? v[q][j - 1] : p)));
          v[q][j] = (i0 + j < m) ? u : (U)0;
        }
      }
      uint32_t w = warp_width(v[q]);
      uint32_t flag = 0;
      if (w == (uint32_t)W) {
        flag = 1;
#pragma unroll
        for (int j = 0; j < K; ++j) v[q][j] = tcms(v[q][j]);
        w = warp_width(v[q]);
      }
      wq[q] = w | (flag << 7);
    }
    // widths → shared ring (2 entries, reused every other chunk), then the
    // chunk size and the aggregate BEFORE waiting for an output slot, so the
    // look-back of later chunks never waits on this CTA's storer
    const uint32_t hb = it & 1;
    if (lane < kSubPerWarp) {
      const uint32_t sub = cw * kSubPerWarp + lane;
      const uint32_t hh = lane == 0 ? wq[0] : lane == 1 ? wq[1] : lane == 2 ? wq[2] : wq[3];
      S.hdr[hb][sub] = (sub * SW < m) ? hh : 0u;
    }
    named_bar_sync(kBarCompute, kCompThreads);
    const uint32_t S_sub = (m + SW - 1) / SW, hdr_bytes = (S_sub + 7) & ~7u;
    const uint32_t h = S.hdr[hb][lane];
    const int32_t rem = (int32_t)m - (int32_t)(lane * SW);
    const uint32_t ms = rem <= 0 ? 0u : (rem < SW ? (uint32_t)rem : (uint32_t)SW);
    const uint32_t b = (ms * (h & 0x7F) + 7) >> 3;
    uint32_t incl = b;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t x = __shfl_up_sync(0xFFFFFFFFu, incl, d);
      if ((int)lane >= d) incl += x;
    }
    const uint32_t total = hdr_bytes + __shfl_sync(0xFFFFFFFFu, incl, 31);
    const uint32_t raw_len = m * (uint32_t)sizeof(U);
    const bool raw = total >= raw_len;  // L104, ties → raw
    const uint32_t len = raw ? raw_len : total;
    if (cw == 0 && lane == 0) {
      lookback_publish(ctx, t, round16(len));
      trace_stamp(a, t, 2);
    }
    mbar_wait(&S.empty_out[o], pho ^ 1);  // output slot free
    if (cw == 0 && lane == 0) trace_stamp(a, t, 3);
    uint8_t* ob = reinterpret_cast<uint8_t*>(S.out[o]);
    if (cw == 0) {
      if (lane == 0) {
        S.out_chunk[o] = t;
        S.out_len[o] = len;
        S.out_raw[o] = raw;
      }
      if (!raw && lane < hdr_bytes) ob[lane] = (uint8_t)h;
    }
    if (raw) {  // store the chunk's own bytes (re-read; L2-resident or HBM)
      const uint4* src = reinterpret_cast<const uint4*>(reinterpret_cast<const uint8_t*>(a.in) + t * kChunkBytes);
      for (uint32_t g = cw * 32 + lane; g < round16(len) / 16; g += kCompThreads) {
        uint4 val;
        if (16 * g + 16 <= len) {
          val = __ldcs(src + g);
        } else {
          const uint32_t* s32 = reinterpret_cast<const uint32_t*>(src + g);
          val.x = s32[0];
          val.y = 16 * g + 4 < len ? s32[1] : 0u;
          val.z = 16 * g + 8 < len ? s32[2] : 0u;
          val.w = 16 * g + 12 < len ? s32[3] : 0u;
        }
        reinterpret_cast<uint4*>(ob)[g] = val;
      }
    } else {
      const uint32_t excl = hdr_bytes + incl - b;  // this lane's subchunk offset
#pragma unroll
      for (int q = 0; q < kSubPerWarp; ++q) {
        const uint32_t sub = cw * kSubPerWarp + q;
        const uint32_t w = wq[q] & 0x7F;
        const uint32_t off = __shfl_sync(0xFFFFFFFFu, excl, sub);
        if (w == 0 || sub >= S_sub) continue;
        const uint32_t L = K * w;
        uint32_t Sg[4];
        make_string(v[q], w, Sg);
        uint32_t* buf = S.out[o] + (off >> 2);
        if (LCF_ENC_OR) {
          emit_or(buf, lane, L, Sg);  // (L < 32 too: a word shared by several lanes takes their ORs)
        } else if (L >= 32) {
          emit_equal(buf, lane, L, Sg);
        } else {
          emit_bits_warp(buf, (uint64_t)lane * L, L, (uint64_t)Sg[0] | ((uint64_t)Sg[1] << 32),
                         (uint64_t)Sg[2] | ((uint64_t)Sg[3] << 32), false, false);
        }
      }
      // zero pad [len, round16(len)): done by the warp owning the last subchunk
      if ((S_sub - 1) / kSubPerWarp == cw) {
        __syncwarp();
        if (lane < 16 && len + lane < round16(len)) ob[len + lane] = 0;
      }
    }
    fence_proxy_async_smem();  // packed bytes → visible to the TMA store
    __syncwarp();
    if (cw == 0 && lane == 0) trace_stamp(a, t, 4);
    if (lane == 0) mbar_arrive(&S.full_out[o]);
  }
}

// (an explicit minimum of 1 block per SM makes ptxas allocate more registers
// than the plain bound, which costs a CTA per SM)
#ifdef LCF_ENC_MINB
#define LCF_ENC_BOUNDS __launch_bounds__(kEncThreads, LCF_ENC_MINB)
#else
#define LCF_ENC_BOUNDS __launch_bounds__(kEncThreads)
#endif
template <typename U>
__global__ void LCF_ENC_BOUNDS speed_encode_kernel(EncArgs a, LaunchCtx ctx) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  EncSmem& S = *reinterpret_cast<EncSmem*>(smem_raw);
  const uint32_t warp = warp_index_uniform(), lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kEncStages; ++i) {
      mbar_init(&S.full_in[i], 1);
      mbar_init(&S.empty_in[i], kCompWarps);
    }
    for (int i = 0; i < kEncOut; ++i) {
      mbar_init(&S.full_out[i], kCompWarps);
      mbar_init(&S.empty_out[i], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (LCF_ENC_OR)  // the output slots start zeroed (then re-zeroed by the storer)
    for (uint32_t i = threadIdx.x; i < sizeof(S.out) / 16; i += blockDim.x)
      reinterpret_cast<uint4*>(&S.out[0][0])[i] = make_uint4(0, 0, 0, 0);
  __syncthreads();
  if (warp == 0) enc_loader<kEncStages>(S, a, ctx, lane, sizeof(U));
  else if (warp <= kStorers) enc_storer<kEncOut, kStorers, EncSmem, false, LCF_ENC_OR>(S, a, ctx, lane, warp - 1);
  else enc_compute<U>(S, a, ctx, warp - 1 - kStorers, lane);
}

// =================================== decode ======================================
template <typename U>
__device__ __forceinline__ void dec_compute(DecSmem<U>& S, const DecArgs& a, const LaunchCtx& ctx, uint32_t cw,
                                            uint32_t lane) {
  using C = Cfg<U>;
  constexpr int W = C::W, CW = C::CW, SW = C::SW, K = C::K;
  const uint4 h0 = reinterpret_cast<const uint4*>(a.stream)[0];
  const uint64_t n_words = (((uint64_t)h0.w << 32) | h0.z) / sizeof(U);
  uint32_t scan_it = 0;
  for (uint32_t it = 0;; ++it) {
    constexpr int kDecStages = DecCfg<U>::kStages;
    const uint32_t s = it % kDecStages, ph = (it / kDecStages) & 1;
    mbar_wait(&S.full_in[s], ph);
    const uint64_t t = S.chunk[s];
    if (t == kNoChunk) return;
    const uint32_t len = S.len[s], fl = S.flags[s];
    const uint32_t m = chunk_words(n_words, t, CW);
    U* dst = reinterpret_cast<U*>(a.out) + t * CW;
    const uint32_t* in = S.in[s];
    if (fl & 2) {  // malformed entry: nothing to decode
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.empty_in[s]);
      continue;
    }
    if (fl & 1) {  // raw chunk: copy
      for (uint32_t g = cw * 32 + lane; g < round16(len) / 16; g += kCompThreads) {
        const uint4 val = reinterpret_cast<const uint4*>(in)[g];
        if (16 * g + 16 <= len) {
          __stcs(reinterpret_cast<uint4*>(dst) + g, val);
        } else {
          const uint32_t wv[4] = {val.x, val.y, val.z, val.w};
          for (int j = 0; j < 4; ++j)
            if (16 * g + 4 * j < len) reinterpret_cast<uint32_t*>(dst)[4 * g + j] = wv[j];
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.empty_in[s]);
      continue;
    }
    // ---- MPLG header: widths, flags, subchunk offsets (L114–118) ----
    const uint32_t S_sub = (m + SW - 1) / SW, hdr_bytes = (S_sub + 7) & ~7u;
    const int32_t rem = (int32_t)m - (int32_t)(lane * SW);
    const uint32_t ms = rem <= 0 ? 0u : (rem < SW ? (uint32_t)rem : (uint32_t)SW);
    uint32_t h = ms ? reinterpret_cast<const uint8_t*>(in)[lane] : 0u;
    const bool badw = (h & 0x7F) > (uint32_t)W;
    if (badw) h = 0;
    const uint32_t b = (ms * (h & 0x7F) + 7) >> 3;
    uint32_t incl = b;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t x = __shfl_up_sync(0xFFFFFFFFu, incl, d);
      if ((int)lane >= d) incl += x;
    }
    const uint32_t total = hdr_bytes + __shfl_sync(0xFFFFFFFFu, incl, 31);
    if (__any_sync(0xFFFFFFFFu, badw) || total != len) {  // every compute warp agrees
      if (cw == 0 && lane == 0) record_error(ctx, DERR_CORRUPT);
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.empty_in[s]);
      continue;
    }
    const uint32_t excl_b = hdr_bytes + incl - b;
    // ---- unpack K fields per lane, unTCMS, differences ----
    U d[kSubPerWarp][K];
    U lane_tot[kSubPerWarp];
#pragma unroll
    for (int q = 0; q < kSubPerWarp; ++q) {
      const uint32_t sub = cw * kSubPerWarp + q;
      const uint32_t hq = __shfl_sync(0xFFFFFFFFu, h, sub);
      const uint32_t off = __shfl_sync(0xFFFFFFFFu, excl_b, sub);
      const uint32_t w = hq & 0x7F;
      const uint32_t P = off * 8 + lane * K * w, F = P >> 5, r = P & 31;
      uint32_t T[5], U4[4];
#pragma unroll
      for (int j = 0; j < 5; ++j) T[j] = in[F + j];  // ≤ 16 B past len: inside the slack, masked off
#pragma unroll
      for (int j = 0; j < 4; ++j) U4[j] = __funnelshift_r(T[j], T[j + 1], r);
      split_string(U4, w, d[q]);
      if (hq >> 7) {  // the TCMS retry (L114, rare): a second inverse; hq is warp-uniform
#pragma unroll
        for (int j = 0; j < K; ++j) d[q][j] = tcms_inv_sx(d[q][j]);
      }
      U tot = 0;
#pragma unroll
      for (int j = 0; j < K; ++j) {
        d[q][j] = tcms_inv_sx(d[q][j]);
        tot += d[q][j];
      }
      lane_tot[q] = tot;
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&S.empty_in[s]);  // stage fully read
    // ---- DIFFMS⁻¹: CTA-wide inclusive prefix sum mod 2^W (L132) ----
    U wcarry = 0, excl_q[kSubPerWarp];
#pragma unroll
    for (int q = 0; q < kSubPerWarp; ++q) {
      U inc = lane_tot[q];
#pragma unroll
      for (int dd = 1; dd < 32; dd <<= 1) {
        const U x = __shfl_up_sync(0xFFFFFFFFu, inc, dd);
        if ((int)lane >= dd) inc += x;
      }
      excl_q[q] = wcarry + inc - lane_tot[q];
      wcarry += shfl_idx(inc, 31);
    }
    const uint32_t sb = scan_it++ & 1;
    if (lane == 0) S.wtot[sb][cw] = wcarry;
    named_bar_sync(kBarCompute, kCompThreads);
    U wbase = 0;
#pragma unroll
    for (uint32_t i = 0; i < kCompWarps; ++i)
      if (i < cw) wbase += S.wtot[sb][i];
#pragma unroll
    for (int q = 0; q < kSubPerWarp; ++q) {
      U run = wbase + excl_q[q];
      U x[K];
#pragma unroll
      for (int j = 0; j < K; ++j) {
        run += d[q][j];
        x[j] = run;
      }
      const uint32_t i0 = (cw * kSubPerWarp + q) * SW + lane * K;
      if (i0 + K <= m) {
        __stcs(reinterpret_cast<uint4*>(dst + i0), pack16<U>(x));
      } else {
#pragma unroll
        for (int j = 0; j < K; ++j)
          if (i0 + j < m) dst[i0 + j] = x[j];
      }
    }
  }
}

#ifdef LCF_DEC_MINB
#define LCF_DEC_BOUNDS __launch_bounds__(kDecThreads, LCF_DEC_MINB)
#else
#define LCF_DEC_BOUNDS __launch_bounds__(kDecThreads, DecCfg<U>::kMinBlocks)
#endif
template <typename U>
__global__ void LCF_DEC_BOUNDS speed_decode_kernel(DecArgs a, LaunchCtx ctx) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  DecSmem<U>& S = *reinterpret_cast<DecSmem<U>*>(smem_raw);
  const uint32_t warp = warp_index_uniform(), lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < DecCfg<U>::kStages; ++i) {
      mbar_init(&S.full_in[i], 1);
      mbar_init(&S.empty_in[i], kCompWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == 0) dec_loader<DecCfg<U>::kStages, kDecBatch>(S, a, ctx, lane, sizeof(U));
  else dec_compute<U>(S, a, ctx, warp - 1, lane);
}

}  // namespace

template <typename U> void launch_speed_encode(const EncArgs& a, const LaunchCtx& ctx, cudaStream_t st) {
  const size_t smem = sizeof(EncSmem);
  static const bool init = [&] {
    cudaFuncSetAttribute(speed_encode_kernel<U>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    return true;
  }();
  (void)init;
  const int grid = persistent_grid(speed_encode_kernel<U>, kEncThreads, smem, a.n_chunks);
  KTrace kt(sizeof(U) == 4 ? "speed_encode_u32" : "speed_encode_u64", st);
  speed_encode_kernel<U><<<grid, kEncThreads, smem, st>>>(a, ctx);
}
template <typename U>
void launch_speed_decode(const DecArgs& a, const LaunchCtx& ctx, uint64_t max_chunks, cudaStream_t st) {
  const size_t smem = sizeof(DecSmem<U>);
  static const bool init = [&] {
    cudaFuncSetAttribute(speed_decode_kernel<U>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    return true;
  }();
  (void)init;
  const int grid = persistent_grid(speed_decode_kernel<U>, kDecThreads, smem, (max_chunks + kDecBatch - 1) / kDecBatch);
  KTrace kt(sizeof(U) == 4 ? "speed_decode_u32" : "speed_decode_u64", st);
  speed_decode_kernel<U><<<grid, kDecThreads, smem, st>>>(a, ctx);
}
template void launch_speed_encode<uint32_t>(const EncArgs&, const LaunchCtx&, cudaStream_t);
template void launch_speed_encode<uint64_t>(const EncArgs&, const LaunchCtx&, cudaStream_t);
template void launch_speed_decode<uint32_t>(const DecArgs&, const LaunchCtx&, uint64_t, cudaStream_t);
template void launch_speed_decode<uint64_t>(const DecArgs&, const LaunchCtx&, uint64_t, cudaStream_t);

}  // namespace lcf
