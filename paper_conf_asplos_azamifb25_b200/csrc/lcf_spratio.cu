// lcf_spratio.cu — SPratio = RZE ∘ BIT₃₂ ∘ DIFFMS₃₂ (§3.2)
// on sm_100a, in the persistent warp-specialised pipeline of lcf_persist.cuh.
//
// Compute threads: 128 (4 warps); thread g owns the 32-word group g of a chunk.
// Encode, per chunk (loader warp, storer warp, one in-place stage):
//   1. a full chunk arrives by a 2-D TMA tensor load into a 128-byte-swizzled
//      stage (row g = group g), so thread g reads its group conflict-free and
//      in word order; DIFFMS (L110–112) in registers
//   2. BIT (L140–142, L162): 32×32 bit transpose in registers (5 butterfly
//      stages, the 16- and 8-bit ones as byte permutes); rows are fed reversed
//      so plane p comes out MSB-first → T[p·G + g] (plane-major)
//   3. RZE (L144–148, L164): byte bitmap B1 of 16-byte units with a packed
//      8-way CTA scan of the unit counts; repetition elimination B1→B2 (CTA
//      scan), B2→B3 and B3→B4 in warp 0 (warp scan, ballot); every section
//      size is known before a byte is written, so the aggregate is published
//      first; then the non-zero and non-repeating bytes are scattered into the
//      stage, which the storer's TMA bulk store reads out.
// Decode inverts the stages from the end of the payload (B4 → B3 → B2 → B1 →
// D), transposes back, runs DIFFMS⁻¹ as a serial per-group scan plus a CTA
// scan of the group totals, and writes a full chunk by a 2-D TMA tensor store
// from a 128-byte-swizzled box.
#include <cuda.h>

#include "lcf_persist.cuh"

namespace lcf {
namespace {

constexpr int kRW = 4;                  // compute warps
constexpr uint32_t kRT = kRW * 32;      // compute threads: one 32-word group each
#ifndef LCF_SPR_STAGES
#define LCF_SPR_STAGES 1  // 1 in-place stage + ≤ 56 registers: 6 CTAs/SM (NYX velocity 452 → 431 µs,
                          // HACC xx 890 → 846 µs); 2 stages at 80 registers: 4 CTAs/SM
#endif
// encode: kRStages input stages, each also the chunk's output buffer (in place)
#ifndef LCF_SPR_DSTAGES
#define LCF_SPR_DSTAGES 1  // 1 stage + ≤ 72 registers: 5 CTAs/SM (measured 420 → 369 µs decode on NYX
                           // velocity on one box, equal on another; 2 stages at 92 registers: 4 CTAs/SM)
#endif
constexpr int kRStages = LCF_SPR_STAGES, kRDecStages = LCF_SPR_DSTAGES, kRDecBatch = 4;
constexpr int kREncThreads = (2 + kRW) * 32, kRDecThreads = (1 + kRW) * 32;
constexpr uint32_t kBarR = 1;           // named barrier of the compute warps

__device__ __forceinline__ void bar_r() { named_bar_sync(kBarR, kRT); }

// ---- 32×32 bit transpose (Hacker's Delight transpose32, fully unrolled) -------
template <int J, uint32_t M> __device__ __forceinline__ void tp_stage(uint32_t (&A)[32]) {
#pragma unroll
  for (int k = 0; k < 32; ++k) {
    if (k & J) continue;
    const uint32_t t = (A[k] ^ (A[k + J] >> J)) & M;
    A[k] ^= t;
    A[k + J] ^= t << J;
  }
}
// The 16- and 8-bit stages move whole bytes: one byte permute per word
// instead of the shift/xor/mask sequence.
template <int J, uint32_t SLO, uint32_t SHI> __device__ __forceinline__ void tp_stage_bytes(uint32_t (&A)[32]) {
#pragma unroll
  for (int k = 0; k < 32; ++k) {
    if (k & J) continue;
    const uint32_t lo = __byte_perm(A[k], A[k + J], SLO), hi = __byte_perm(A[k], A[k + J], SHI);
    A[k] = lo;
    A[k + J] = hi;
  }
}
// A[i] = row i with column c at bit 31−c  →  A'[c] bit (31−i) = A[i] bit (31−c)
__device__ __forceinline__ void transpose32(uint32_t (&A)[32]) {
  tp_stage_bytes<16, 0x3276u, 0x1054u>(A);  // ≡ tp_stage<16, 0x0000FFFF>
  tp_stage_bytes<8, 0x3715u, 0x2604u>(A);   // ≡ tp_stage<8, 0x00FF00FF>
  tp_stage<4, 0x0F0F0F0Fu>(A);
  tp_stage<2, 0x33333333u>(A);
  tp_stage<1, 0x55555555u>(A);
}

// 4-bit mask of the non-zero bytes of w (bit b ↔ byte b)
__device__ __forceinline__ uint32_t nz_nibble(uint32_t w) {
  const uint32_t t = (((w & 0x7F7F7F7Fu) + 0x7F7F7F7Fu) | w) & 0x80808080u;
  return (t * 0x00204081u) >> 28;
}
__device__ __forceinline__ uint32_t nz_mask16(const uint4& q) {
  return nz_nibble(q.x) | (nz_nibble(q.y) << 4) | (nz_nibble(q.z) << 8) | (nz_nibble(q.w) << 12);
}

// Exclusive scan over the 128 compute threads; `sh` is a 4-entry slot used
// once per chunk (reuse is separated by later barriers).
template <typename T>
__device__ __forceinline__ T cta_excl_scan(T v, T* sh, uint32_t cw, uint32_t lane, T& total) {
  T x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const T y = __shfl_up_sync(0xFFFFFFFFu, x, d);
    if ((int)lane >= d) x += y;
  }
  if (lane == 31) sh[cw] = x;
  bar_r();
  T base = 0;
  total = 0;
#pragma unroll
  for (uint32_t i = 0; i < kRW; ++i) {
    const T s = sh[i];
    if (i < cw) base += s;
    total += s;
  }
  return base + x - v;
}

struct RZESizes {
  uint32_t L, L1, L2, L3, L4;
};
__device__ __forceinline__ RZESizes rze_sizes(uint32_t L) {
  RZESizes z;
  z.L = L;
  z.L1 = (L + 7) / 8;
  z.L2 = (z.L1 + 7) / 8;
  z.L3 = (z.L2 + 7) / 8;
  z.L4 = (z.L3 + 7) / 8;
  return z;
}

struct REncSmem {
  // raw chunk, then its encoding. A full chunk arrives by a 2-D TMA tensor load
  // as 128 rows of 128 bytes (one 32-word group per row) in the 128-byte
  // swizzle — 16-byte piece q of row g at q ^ (g mod 8), so that every thread
  // reads its own group conflict-free and in word order; a ragged chunk by a
  // 1-D copy in plain order (in_swz)
  alignas(1024) uint32_t in[kRStages][4096];
  alignas(128) uint32_t T[4096];  // BIT output = RZE input D
  alignas(16) uint8_t B1[2048 + 16];
  alignas(16) uint8_t B2[256 + 16];
  uint64_t full_in[kRStages], empty_in[kRStages], full_out[kRStages];
  uint64_t in_chunk[kRStages], out_chunk[kRStages];
  uint32_t out_len[kRStages], out_raw[kRStages], in_swz[kRStages];
  uint64_t sc64[2][kRW];
  uint32_t sc32[2][kRW];
  uint32_t b3;  // B3 bytes (≤ 32), kept by warp 0 in registers; B4 here
};

struct RDecSmem {
  alignas(128) uint32_t in[kRDecStages][(kChunkBytes + 64) / 4];
  // T: decoded D (plane-major, 4096 words), then — once every thread holds its
  // group in registers — the decoded words with a 33-word row stride (X)
  alignas(1024) uint32_t T[kRT * 33];  // (1024-aligned: the 128-byte swizzle of the output box)
  alignas(16) uint8_t B1[2048 + 16];
  alignas(16) uint8_t B2[256 + 16];
  uint64_t full_in[kRDecStages], empty_in[kRDecStages];
  uint64_t chunk[kRDecStages];
  uint32_t len[kRDecStages], flags[kRDecStages];
  uint64_t sc64[2][kRW];
  uint32_t sc32[3][kRW];
  uint32_t xsel[16];  // __byte_perm selectors: byte j ← source byte #(set bits of m below j) if bit j of m, else 0
  int32_t s2, bad;
};

// =================================== encode ======================================
__device__ __forceinline__ void r_enc_compute(REncSmem& S, const EncArgs& a, const LaunchCtx& ctx, uint32_t cw,
                                              uint32_t lane) {
  const uint32_t g = cw * 32 + lane;  // this thread's group
  for (uint32_t it = 0;; ++it) {
    const uint32_t s = it % kRStages, ph = (it / kRStages) & 1;
    mbar_wait(&S.full_in[s], ph);
    const uint64_t t = S.in_chunk[s];
    if (t == kNoChunk) {  // the stage is ours: forward the end marker through it
      if (cw == 0 && lane == 0) S.out_chunk[s] = kNoChunk;
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.full_out[s]);
      return;
    }
    if (g == 0) trace_stamp(a, t, 1);
    const uint32_t m = chunk_words(a.n_words_total, a.first_chunk + t, 4096);
    const uint32_t G = m / 32;  // full groups; m mod 32 leftover words are copied (A-9)
    const uint32_t* in = S.in[s];

    // ---- 1. DIFFMS (L110–112), 2. BIT (L140–142) ----
    const bool swz = S.in_swz[s];
    if (g < G) {
      uint32_t A[32];
#pragma unroll
      for (int q = 0; q < 8; ++q) {  // words 32g + 4q …: piece q of row g (swizzled: conflict-free)
        const uint4 v = reinterpret_cast<const uint4*>(in)[8 * g + (swz ? (q ^ (g & 7)) : q)];
        A[4 * q] = v.x; A[4 * q + 1] = v.y; A[4 * q + 2] = v.z; A[4 * q + 3] = v.w;
      }
      const uint32_t r = g - 1;  // word 32g − 1: last word of row g − 1
      const uint32_t xprev = g ? in[32 * r + 4 * (swz ? (7 ^ (r & 7)) : 7) + 3] : 0u;
#pragma unroll
      for (int j = 31; j >= 0; --j) A[j] = tcms(A[j] - (j ? A[j - 1] : xprev));
#pragma unroll
      for (int i = 0; i < 16; ++i) {  // rows reversed → planes MSB-first
        const uint32_t tmp = A[i];
        A[i] = A[31 - i];
        A[31 - i] = tmp;
      }
      transpose32(A);
#pragma unroll
      for (int p = 0; p < 32; ++p) S.T[p * G + g] = A[p];
    } else if (g == G && (m & 31)) {  // leftover words: DIFFMS, copied unchanged by BIT
      for (uint32_t i = 32 * G; i < m; ++i) S.T[i] = tcms(in[i] - (i ? in[i - 1] : 0u));
    }
    const RZESizes z = rze_sizes(4 * m);
    const uint32_t NU = (z.L + 15) / 16;  // 16-byte units of D
    if (m < 4096) {  // ragged chunk: zero D beyond L and the bitmap tails
      for (uint32_t i = m + g; i < 4096; i += kRT) S.T[i] = 0;
      for (uint32_t i = g; i < (2048 + 16) / 4; i += kRT) reinterpret_cast<uint32_t*>(S.B1)[i] = 0;
    }
    bar_r();  // the stage has been read: from here on it is the output buffer

    // ---- 3. RZE (L144–148): B1 and counts of the units u = g + 128k ----
    uint64_t pk[2] = {0, 0};
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const uint32_t u = g + kRT * k;
      if (u < NU) {
        const uint32_t mk = nz_mask16(reinterpret_cast<const uint4*>(S.T)[u]);
        reinterpret_cast<uint16_t*>(S.B1)[u] = (uint16_t)mk;
        pk[k >> 2] |= (uint64_t)__popc(mk) << (16 * (k & 3));
      }
    }
    uint64_t tot0, tot1;
    const uint64_t ex0 = cta_excl_scan<uint64_t>(pk[0], S.sc64[0], cw, lane, tot0);
    const uint64_t ex1 = cta_excl_scan<uint64_t>(pk[1], S.sc64[1], cw, lane, tot1);
    uint32_t nnzD = 0, koff[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const uint64_t tk = (k < 4 ? tot0 : tot1) >> (16 * (k & 3)) & 0xFFFF;
      koff[k] = nnzD + (uint32_t)(((k < 4 ? ex0 : ex1) >> (16 * (k & 3))) & 0xFFFF);
      nnzD += (uint32_t)tk;
    }
    // B1 → B2 (bytes [16g, 16g+16) of B1), repetition elimination (L146)
    uint32_t c1 = 0;
    uint4 b1v = make_uint4(0, 0, 0, 0);
    if (16 * g < z.L1) {
      b1v = reinterpret_cast<const uint4*>(S.B1)[g];
      const uint32_t prev = g ? S.B1[16 * g - 1] : 0u;
      const uint32_t w[4] = {b1v.x, b1v.y, b1v.z, b1v.w};
#pragma unroll
      for (int j = 0; j < 16; ++j) {
        const uint32_t cur = (w[j >> 2] >> (8 * (j & 3))) & 0xFF;
        const uint32_t pre = j ? (w[(j - 1) >> 2] >> (8 * ((j - 1) & 3))) & 0xFF : prev;
        if (cur != pre && 16 * g + j < z.L1) c1 |= 1u << j;
      }
      reinterpret_cast<uint16_t*>(S.B2)[g] = (uint16_t)c1;
    } else if (2 * g < 256 + 16) {
      reinterpret_cast<uint16_t*>(S.B2)[g] = 0;
    }
    uint32_t nr1;
    const uint32_t off1 = cta_excl_scan<uint32_t>(__popc(c1), S.sc32[0], cw, lane, nr1);
    // B2 → B3 → B4 in warp 0 (L2 ≤ 256 bytes, L3 ≤ 32 bytes)
    uint32_t nr2 = 0, nr3 = 0, b3 = 0, c2 = 0, off2 = 0, b2w0 = 0, b2w1 = 0, b4 = 0;
    if (cw == 0) {
      // lane handles B2 bytes [8·lane, 8·lane+8)
      b2w0 = reinterpret_cast<const uint32_t*>(S.B2)[2 * lane];
      b2w1 = reinterpret_cast<const uint32_t*>(S.B2)[2 * lane + 1];
      const uint32_t prevb = __shfl_up_sync(0xFFFFFFFFu, b2w1 >> 24, 1);
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint32_t cur = ((j < 4 ? b2w0 : b2w1) >> (8 * (j & 3))) & 0xFF;
        const uint32_t pre = j ? (((j - 1) < 4 ? b2w0 : b2w1) >> (8 * ((j - 1) & 3))) & 0xFF : (lane ? prevb : 0u);
        if (cur != pre && 8 * lane + j < z.L2) c2 |= 1u << j;
      }
      b3 = c2;  // B3 byte `lane`
      uint32_t x = __popc(c2);
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
        if ((int)lane >= d) x += y;
      }
      off2 = x - __popc(c2);
      nr2 = __shfl_sync(0xFFFFFFFFu, x, 31);
      const uint32_t pb3 = __shfl_up_sync(0xFFFFFFFFu, b3, 1);
      const bool ch3 = lane < z.L3 && b3 != (lane ? pb3 : 0u);
      b4 = __ballot_sync(0xFFFFFFFFu, ch3);
      nr3 = __popc(b4);
    }
    // totals: every thread needs the final length; warp 0 broadcasts through smem
    if (cw == 0 && lane == 0) S.sc32[1][0] = nr2 | (nr3 << 16);
    bar_r();
    {
      const uint32_t v = S.sc32[1][0];
      nr2 = v & 0xFFFF;
      nr3 = v >> 16;
    }
    const uint32_t total = nnzD + nr1 + nr2 + nr3 + z.L4;
    const uint32_t raw_len = 4 * m;
    const bool raw = total >= raw_len;  // L104, ties → raw
    const uint32_t len = raw ? raw_len : total;
    if (cw == 0 && lane == 0) {
      lookback_publish(ctx, t, round16(len));
      trace_stamp(a, t, 2);
    }
    if (g == 0) trace_stamp(a, t, 3);
    if (cw == 0 && lane == 0) {
      S.out_chunk[s] = t;
      S.out_len[s] = len;
      S.out_raw[s] = raw;
    }
    uint8_t* ob = reinterpret_cast<uint8_t*>(S.in[s]);
    if (raw) {  // the stage still holds the raw chunk: zero its padding
      if (swz) {  // (a full chunk, swizzled in the stage: its bytes again, from L2 / HBM)
        const uint4* src = reinterpret_cast<const uint4*>(reinterpret_cast<const uint8_t*>(a.in) + t * kChunkBytes);
        for (uint32_t q = g; q < kChunkBytes / 16; q += kRT) reinterpret_cast<uint4*>(ob)[q] = __ldcg(src + q);
      }
      if (g < round16(len) - len) ob[len + g] = 0;
    } else {
      // nz(D): non-zero bytes of every unit at its scanned offset
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const uint32_t u = g + kRT * k;
        if (u >= NU) continue;
        const uint4 v = reinterpret_cast<const uint4*>(S.T)[u];
        const uint32_t w[4] = {v.x, v.y, v.z, v.w};
        uint32_t p = koff[k];
#pragma unroll
        for (int b = 0; b < 16; ++b) {
          const uint32_t by = (w[b >> 2] >> (8 * (b & 3))) & 0xFF;
          if (by) ob[p++] = (uint8_t)by;
        }
      }
      // nr(B1)
      {
        uint32_t p = nnzD + off1;
        const uint32_t w[4] = {b1v.x, b1v.y, b1v.z, b1v.w};
#pragma unroll
        for (int j = 0; j < 16; ++j)
          if ((c1 >> j) & 1) ob[p++] = (uint8_t)(w[j >> 2] >> (8 * (j & 3)));
      }
      if (cw == 0) {
        // nr(B2), nr(B3), B4
        uint32_t p = nnzD + nr1 + off2;
#pragma unroll
        for (int j = 0; j < 8; ++j)
          if ((c2 >> j) & 1) ob[p++] = (uint8_t)((j < 4 ? b2w0 : b2w1) >> (8 * (j & 3)));
        if ((b4 >> lane) & 1) ob[nnzD + nr1 + nr2 + __popc(b4 & ((1u << lane) - 1))] = (uint8_t)b3;
        if (lane < z.L4) ob[total - z.L4 + lane] = (uint8_t)(b4 >> (8 * lane));
        if (lane < 16 && total + lane < round16(total)) ob[total + lane] = 0;
      }
    }
    fence_proxy_async_smem();
    __syncwarp();
    if (g == 0) trace_stamp(a, t, 4);
    if (lane == 0) mbar_arrive(&S.full_out[s]);
    bar_r();  // T, B1, B2 and the scan slots are rewritten by the next chunk
  }
}

// The loader: as enc_loader (lcf_persist.cuh), but a full chunk comes as one
// 2-D TMA tensor load of its 128 × 128-byte box into the swizzled stage.
__device__ __forceinline__ void r_enc_loader(REncSmem& S, const EncArgs& a, const LaunchCtx& ctx, uint32_t lane,
                                             const CUtensorMap* tmap) {
  for (uint32_t it = 0;; ++it) {
    const uint32_t s = it % kRStages, ph = (it / kRStages) & 1;
    mbar_wait(&S.empty_in[s], ph ^ 1);
    uint64_t t = 0;
    if (lane == 0) t = atomicAdd(ctx.ticket, 1ull);
    t = __shfl_sync(0xFFFFFFFFu, t, 0);
    if (t >= a.n_chunks) {
      if (lane == 0) {
        S.in_chunk[s] = kNoChunk;
        mbar_arrive(&S.full_in[s]);
        ticket_retire(ctx);
      }
      return;
    }
    const uint32_t bytes = chunk_words(a.n_words_total, a.first_chunk + t, 4096) * 4;
    const uint8_t* src = reinterpret_cast<const uint8_t*>(a.in) + t * kChunkBytes;
    if (lane == 0) trace_stamp(a, t, 0);
    if (tmap && bytes == kChunkBytes) {
      if (lane == 0) {
        S.in_chunk[s] = t;
        S.in_swz[s] = 1;
        mbar_arrive_expect_tx(&S.full_in[s], kChunkBytes);
        tma_load_2d(S.in[s], tmap, 0, (int32_t)(t * 128), &S.full_in[s]);
      }
    } else if ((bytes & 15) == 0) {
      if (lane == 0) {
        S.in_chunk[s] = t;
        S.in_swz[s] = 0;
        mbar_arrive_expect_tx(&S.full_in[s], bytes);
        tma_load_1d(S.in[s], src, bytes, &S.full_in[s]);
      }
    } else {  // ragged tail chunk: plain loads
      for (uint32_t i = lane; i < bytes / 4; i += 32) S.in[s][i] = reinterpret_cast<const uint32_t*>(src)[i];
      if (lane == 0) {
        S.in_chunk[s] = t;
        S.in_swz[s] = 0;
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.full_in[s]);
    }
  }
}

// A [rows][32 u32] tensor map over `base` for 2-D TMA boxes of 128 rows in the
// 128-byte swizzle (cuTensorMapEncodeTiled from the driver at run time, so the
// library needs no link-time libcuda); false if unavailable.
static bool rows_tensor_map(CUtensorMap* tm, const void* base, uint64_t rows) {
  typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                               const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                               CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
  static EncodeFn encode = [] {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      fn = nullptr;
    return reinterpret_cast<EncodeFn>(fn);
  }();
  memset(tm, 0, sizeof(*tm));
  if (!encode || rows < 128 || rows >= (1ull << 31) || ((uintptr_t)base & 15)) return false;
  const cuuint64_t dims[2] = {32, rows}, strides[1] = {128};
  const cuuint32_t box[2] = {32, 128}, es[2] = {1, 1};
  return encode(tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, const_cast<void*>(base), dims, strides, box, es,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

#ifndef LCF_SPR_TMA_IN
#define LCF_SPR_TMA_IN 1
#endif
#ifndef LCF_SPR_ENC_WU
#define LCF_SPR_ENC_WU 0  // the uniform warp index (no convergence wrappers) measured 1 % slower here
#endif
#ifndef LCF_SPR_ENC_MINB
#define LCF_SPR_ENC_MINB 6
#endif
__global__ void __launch_bounds__(kREncThreads, LCF_SPR_ENC_MINB)
    spratio_encode_kernel(EncArgs a, LaunchCtx ctx, const __grid_constant__ CUtensorMap tmap, uint32_t use_tmap) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  REncSmem& S = *reinterpret_cast<REncSmem*>(smem_raw);
  const uint32_t warp = LCF_SPR_ENC_WU ? warp_index_uniform() : threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kRStages; ++i) {
      mbar_init(&S.full_in[i], 1);
      mbar_init(&S.empty_in[i], 1);  // released by the storer
      mbar_init(&S.full_out[i], kRW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  // (the swizzled box needs a 1024-byte aligned stage: otherwise 1-D copies)
  const bool tma = use_tmap && (smem_addr(S.in[0]) & 1023) == 0;
  if (warp == 0) r_enc_loader(S, a, ctx, lane, tma ? &tmap : nullptr);
  else if (warp == 1) enc_storer<kRStages, 1, REncSmem, true>(S, a, ctx, lane, 0);
  else r_enc_compute(S, a, ctx, warp - 2, lane);
}

// =================================== decode ======================================
// Output of a full chunk (LCF_SPR_TMA_OUT): thread g writes its group's 32
// decoded words as row g of a 128 × 128-byte box in S.T, 16-byte piece q at
// q ^ (g mod 8) (the 128-byte swizzle: conflict-free, no register shuffling),
// and one thread stores the box with a 2-D TMA tensor store that un-swizzles
// it into 16 KiB of contiguous output. Ragged chunks keep the thread stores.
#ifndef LCF_SPR_TMA_OUT
#define LCF_SPR_TMA_OUT 1
#endif
__device__ __forceinline__ void r_dec_compute(RDecSmem& S, const DecArgs& a, const LaunchCtx& ctx, uint32_t cw,
                                              uint32_t lane, const CUtensorMap* tmap) {
  const uint32_t g = cw * 32 + lane;
  const uint4 h0 = reinterpret_cast<const uint4*>(a.stream)[0];
  const uint64_t n_words = (((uint64_t)h0.w << 32) | h0.z) / 4;
  for (uint32_t it = 0;; ++it) {
    const uint32_t s = it % kRDecStages, ph = (it / kRDecStages) & 1;
    mbar_wait(&S.full_in[s], ph);
    const uint64_t t = S.chunk[s];
    if (t == kNoChunk) {
      if (g == 0) tma_store_wait_all0();  // the last box has left S.T
      return;
    }
    const uint32_t len = S.len[s], fl = S.flags[s];
    const uint32_t m = chunk_words(n_words, t, 4096);
    uint32_t* dst = reinterpret_cast<uint32_t*>(a.out) + t * 4096;
    const uint8_t* in = reinterpret_cast<const uint8_t*>(S.in[s]);
    if (fl & 2) {
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.empty_in[s]);
      continue;
    }
    if (fl & 1) {  // raw chunk: copy
      for (uint32_t q = g; q < round16(len) / 16; q += kRT) {
        const uint4 val = reinterpret_cast<const uint4*>(in)[q];
        if (16 * q + 16 <= len) {
          __stcs(reinterpret_cast<uint4*>(dst) + q, val);
        } else {
          const uint32_t wv[4] = {val.x, val.y, val.z, val.w};
          for (int j = 0; j < 4; ++j)
            if (16 * q + 4 * j < len) dst[4 * q + j] = wv[j];
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.empty_in[s]);
      continue;
    }
    const RZESizes z = rze_sizes(4 * m);
    const uint32_t G = m / 32, NU = (z.L + 15) / 16;
    // ---- RZE⁻¹ from the end: B4 → B3 → B2 (warp 0) ----
    if (cw == 0) {
      int32_t bad = len < z.L4;
      uint32_t b4 = 0;
      if (!bad)
        for (uint32_t i = 0; i < z.L4; ++i) b4 |= (uint32_t)in[len - z.L4 + i] << (8 * i);
      const uint32_t v3 = z.L3 >= 32 ? 0xFFFFFFFFu : ((1u << z.L3) - 1u);
      const int32_t s3 = (int32_t)len - (int32_t)z.L4 - __popc(b4 & v3);
      if (s3 < 0) bad = 1;
      const uint32_t r3 = __popc(b4 & v3 & (0xFFFFFFFFu >> (31 - lane)));
      const uint32_t b3 = (!bad && lane < z.L3 && r3) ? in[s3 + r3 - 1] : 0u;  // B3 byte `lane`
      // B2 bytes [8·lane, 8·lane+8): bits of B3 byte `lane`
      const uint32_t vb = (8 * lane >= z.L2) ? 0u : (z.L2 - 8 * lane >= 8 ? 0xFFu : ((1u << (z.L2 - 8 * lane)) - 1u));
      const uint32_t bits2 = b3 & vb;
      uint32_t x = __popc(bits2);
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
        if ((int)lane >= d) x += y;
      }
      const uint32_t cnt2 = __shfl_sync(0xFFFFFFFFu, x, 31);
      const int32_t s2 = s3 - (int32_t)cnt2;
      if (s2 < 0) bad = 1;
      bad = __any_sync(0xFFFFFFFFu, bad);
      uint32_t r = x - __popc(bits2);
      uint32_t wv[2] = {0, 0};
      // rank r counts set bits before byte j; value = nr2[r−1] of the last set bit
      const uint32_t prev_r = r;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        r += (bits2 >> j) & 1;
        const uint32_t val = (!bad && r) ? in[s2 + r - 1] : 0u;
        wv[j >> 2] |= val << (8 * (j & 3));
      }
      (void)prev_r;
      reinterpret_cast<uint32_t*>(S.B2)[2 * lane] = wv[0];
      reinterpret_cast<uint32_t*>(S.B2)[2 * lane + 1] = wv[1];
      if (lane == 0) {
        S.s2 = s2;
        S.bad = bad;
      }
      if (lane == 0) tma_store_wait_read0();  // the previous chunk's box has been read out of S.T
    }
    bar_r();
    int32_t bad = S.bad;
    const int32_t s2 = S.s2;
    // ---- B1: bytes [16g, 16g+16), bits = B2 bytes 2g, 2g+1 ----
    uint32_t bits1 = 0;
    if (16 * g < z.L1) {
      bits1 = reinterpret_cast<const uint16_t*>(S.B2)[g];
      const uint32_t nvalid = z.L1 - 16 * g;
      if (nvalid < 16) bits1 &= (1u << nvalid) - 1u;
    }
    uint32_t cnt1;
    uint32_t r1 = cta_excl_scan<uint32_t>(__popc(bits1), S.sc32[0], cw, lane, cnt1);
    const int32_t s1 = s2 - (int32_t)cnt1;
    if (s1 < 0) bad = 1;
    if (16 * g < 2048 + 16) {
      uint32_t wv[4] = {0, 0, 0, 0};
      if (!bad) {
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          r1 += (bits1 >> j) & 1;
          const uint32_t val = r1 ? in[s1 + r1 - 1] : 0u;
          wv[j >> 2] |= val << (8 * (j & 3));
        }
      }
      if (16 * g < z.L1) reinterpret_cast<uint4*>(S.B1)[g] = make_uint4(wv[0], wv[1], wv[2], wv[3]);
    }
    bar_r();
    // ---- D: units u = g + 128k, bits = B1 bytes 2u, 2u+1 ----
    uint32_t ub[8];
    uint64_t pk[2] = {0, 0};
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const uint32_t u = g + kRT * k;
      ub[k] = 0;
      if (u < NU) {
        ub[k] = reinterpret_cast<const uint16_t*>(S.B1)[u];
        const uint32_t nvalid = z.L - 16 * u;
        if (nvalid < 16) ub[k] &= (1u << nvalid) - 1u;
        pk[k >> 2] |= (uint64_t)__popc(ub[k]) << (16 * (k & 3));
      }
    }
    uint64_t tot0, tot1;
    const uint64_t ex0 = cta_excl_scan<uint64_t>(pk[0], S.sc64[0], cw, lane, tot0);
    const uint64_t ex1 = cta_excl_scan<uint64_t>(pk[1], S.sc64[1], cw, lane, tot1);
    uint32_t nnz = 0, koff[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      koff[k] = nnz + (uint32_t)(((k < 4 ? ex0 : ex1) >> (16 * (k & 3))) & 0xFFFF);
      nnz += (uint32_t)(((k < 4 ? tot0 : tot1) >> (16 * (k & 3))) & 0xFFFF);
    }
    if ((int32_t)nnz != s1) bad = 1;  // nz(D) must end where nr(B1) starts
    if (bad) {  // every compute thread reached the same verdict from the same smem data
      if (g == 0) record_error(ctx, DERR_CORRUPT);
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.empty_in[s]);
      bar_r();  // keep the barrier count of every compute warp in step
      continue;
    }
    // expand: word wi of the unit takes popc(m) bytes from nz(D) at p
    // (one unaligned 4-byte read = two words + a funnel shift) and spreads them
    // to its set byte positions with one byte permute (S.xsel[m])
    const uint32_t* in32 = reinterpret_cast<const uint32_t*>(in);
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const uint32_t u = g + kRT * k;
      if (u >= NU) continue;
      uint32_t wv[4], p = koff[k];
#pragma unroll
      for (int wi = 0; wi < 4; ++wi) {
        const uint32_t m = (ub[k] >> (4 * wi)) & 0xFu;
        const uint32_t q = p >> 2;
        const uint32_t src = __funnelshift_r(in32[q], in32[q + 1], 8 * (p & 3));
        wv[wi] = __byte_perm(src, 0u, S.xsel[m]);
        p += __popc(m);
      }
      reinterpret_cast<uint4*>(S.T)[u] = make_uint4(wv[0], wv[1], wv[2], wv[3]);
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&S.empty_in[s]);  // payload fully consumed
    bar_r();
    // ---- BIT⁻¹ (rows out reversed) and DIFFMS⁻¹ (serial + CTA scan) ----
    uint32_t X[32];
    uint32_t tot = 0;
    if (g < G) {
#pragma unroll
      for (int p = 0; p < 32; ++p) X[p] = S.T[p * G + g];
      transpose32(X);
#pragma unroll
      for (int i = 0; i < 16; ++i) {  // U[i] = A'[31−i]
        const uint32_t tmp = X[i];
        X[i] = X[31 - i];
        X[31 - i] = tmp;
      }
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        tot += tcms_inv(X[i]);
        X[i] = tot;
      }
    } else if (g == G && (m & 31)) {  // leftover words (A-9): DIFFMS⁻¹ only
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        if ((uint32_t)i < (m & 31)) tot += tcms_inv(S.T[32 * G + i]);
        X[i] = tot;
      }
    }
    uint32_t all;
    // the scan's barrier also ends every read of T: X overwrites it below
    const uint32_t base = cta_excl_scan<uint32_t>(tot, S.sc32[1], cw, lane, all);
    uint32_t* const Xs = S.T;
    if (tmap && m == 4096) {
      uint8_t* row = reinterpret_cast<uint8_t*>(S.T) + 128 * g;
#pragma unroll
      for (uint32_t q = 0; q < 8; ++q)
        *reinterpret_cast<uint4*>(row + 16 * (q ^ (g & 7))) =
            make_uint4(X[4 * q] + base, X[4 * q + 1] + base, X[4 * q + 2] + base, X[4 * q + 3] + base);
      fence_proxy_async_smem();
      bar_r();
      if (g == 0) {
        tma_store_2d(tmap, S.T, 0, (int32_t)(t * 128));
        tma_store_commit();
      }
      continue;
    }
    if (g < G || (g == G && (m & 31))) {
#pragma unroll
      for (int i = 0; i < 32; ++i) Xs[g * 33 + i] = X[i] + base;
    }
    bar_r();
    // coalesced 16-byte stores of words n = 4q .. 4q+3
    for (uint32_t q = g; q < 1024; q += kRT) {
      const uint32_t n = 4 * q;
      if (n >= m) break;
      const uint32_t* row = Xs + (n >> 5) * 33 + (n & 31);
      if (n + 4 <= m) {
        __stcs(reinterpret_cast<uint4*>(dst) + q, make_uint4(row[0], row[1], row[2], row[3]));
      } else {
        for (uint32_t j = 0; n + j < m; ++j) dst[n + j] = row[j];
      }
    }
  }
}

#ifndef LCF_SPR_DEC_MINB
#define LCF_SPR_DEC_MINB 6  // 64 registers, no spills since the warp-uniform dispatch: 6 CTAs/SM (NYX velocity 324 -> 304 us)
#endif
__global__ void __launch_bounds__(kRDecThreads, LCF_SPR_DEC_MINB)
    spratio_decode_kernel(DecArgs a, LaunchCtx ctx, const __grid_constant__ CUtensorMap tmap, uint32_t use_tmap) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  RDecSmem& S = *reinterpret_cast<RDecSmem*>(smem_raw);
  const uint32_t warp = warp_index_uniform(), lane = threadIdx.x & 31;
  if (threadIdx.x < 16) {
    const uint32_t m = threadIdx.x;
    uint32_t sel = 0, c = 0;
    for (int j = 0; j < 4; ++j) {
      sel |= (((m >> j) & 1u) ? c : 4u) << (4 * j);
      c += (m >> j) & 1u;
    }
    S.xsel[m] = sel;
  }
  if (threadIdx.x == 0) {
    for (int i = 0; i < kRDecStages; ++i) {
      mbar_init(&S.full_in[i], 1);
      mbar_init(&S.empty_in[i], kRW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == 0) dec_loader<kRDecStages, kRDecBatch>(S, a, ctx, lane, 4);
  // (the swizzled box needs a 1024-byte aligned S.T: otherwise thread stores)
  const bool tma = use_tmap && (smem_addr(S.T) & 1023) == 0;
  if (warp != 0) r_dec_compute(S, a, ctx, warp - 1, lane, tma ? &tmap : nullptr);
}

}  // namespace

void launch_spratio_encode(const EncArgs& a, const LaunchCtx& ctx, cudaStream_t st) {
  const size_t smem = sizeof(REncSmem);
  static const bool init = [&] {
    cudaFuncSetAttribute(spratio_encode_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    return true;
  }();
  (void)init;
  const int grid = persistent_grid(spratio_encode_kernel, kREncThreads, smem, a.n_chunks);
  // full chunks of this launch (only the stream's last chunk can be ragged)
  const uint64_t full = (a.first_chunk + a.n_chunks) * 4096 <= a.n_words_total ? a.n_chunks : a.n_chunks - 1;
  CUtensorMap tm;
  const uint32_t use = LCF_SPR_TMA_IN && rows_tensor_map(&tm, a.in, full * 128);
  KTrace kt("spratio_encode", st);
  spratio_encode_kernel<<<grid, kREncThreads, smem, st>>>(a, ctx, tm, use);
}

void launch_spratio_decode(const DecArgs& a, const LaunchCtx& ctx, uint64_t max_chunks, cudaStream_t st) {
  const size_t smem = sizeof(RDecSmem);
  static const bool init = [&] {
    cudaFuncSetAttribute(spratio_decode_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    return true;
  }();
  (void)init;
  const int grid = persistent_grid(spratio_decode_kernel, kRDecThreads, smem, (max_chunks + kRDecBatch - 1) / kRDecBatch);
  // the output as a [rows][32 words] tensor for the 2-D TMA stores of full chunks
  CUtensorMap tm;
  const uint32_t use = LCF_SPR_TMA_OUT && rows_tensor_map(&tm, a.out, a.out_capacity / 128);
  KTrace kt("spratio_decode", st);
  spratio_decode_kernel<<<grid, kRDecThreads, smem, st>>>(a, ctx, tm, use);
}

}  // namespace lcf
