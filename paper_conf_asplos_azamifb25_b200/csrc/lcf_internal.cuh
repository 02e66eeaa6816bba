// lcf_internal.cuh — device-side building blocks shared by the sm_100a codec
// kernels: stream constants (FORMAT.md), decoupled look-back (Merrill &
// Garland, PAPER.md L122 ref [28]), warp bit-string emission, word helpers.
// Nothing here is shared with oracle/.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace lcf {

// ---- stream constants (FORMAT.md §1) ---------------------------------------
constexpr uint32_t kMagic = 0x3146434Cu;  // "LCF1"
constexpr uint32_t kVersion = 1;
constexpr uint32_t kHeaderBytes = 32;
constexpr uint32_t kChunkBytes = 16384;  // L104
constexpr uint32_t kRawFlag = 0x80000000u;

enum Algo : int { SPSPEED = 0, SPRATIO = 1, DPSPEED = 2, DPRATIO = 3 };

// Error bits recorded by device code in the workspace error word, which holds
// max over failing launches of (epoch << 8 | bits): the newest failure wins.
enum DevErr : uint32_t { DERR_CORRUPT = 1u, DERR_SMALL = 2u };

__host__ __device__ constexpr uint64_t round16(uint64_t v) { return (v + 15) & ~uint64_t(15); }

struct StreamHeader {  // 32 bytes, little-endian (FORMAT.md §1)
  uint32_t magic;
  uint8_t version, algo, word_bytes, zero;
  uint64_t n_bytes, n_chunks, payload_bytes;
};
static_assert(sizeof(StreamHeader) == 32, "header layout");

// ---- launch context shared by all chunk kernels ----------------------------
struct LaunchCtx {
  unsigned long long* ticket;  // [0] tickets handed out, [1] retired CTAs (reset by the last)
  uint64_t* status;            // look-back status words, one per chunk
  uint32_t epoch;              // 1 .. 2^22-1, unique per launch between resets
  uint32_t* err;               // device error word
};

// ---- relaxed/acquire/release global accesses -------------------------------
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// system scope: words of peer GPUs mapped through CUDA IPC (NVLink)
__device__ __forceinline__ uint64_t ld_relaxed_sys_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_sys_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_sys_u64(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_cg_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void record_error(const LaunchCtx& ctx, uint32_t bits) {
  atomicMax(ctx.err, (ctx.epoch << 8) | bits);
}

// ---- decoupled look-back (single-pass scan of chunk sizes, L120–122) -------
// status word: [63:62] flag (1 aggregate, 2 inclusive) | [61:40] epoch | [39:0] value
constexpr uint64_t kFlagAgg = 1, kFlagInc = 2;
__device__ __forceinline__ uint64_t make_status(uint64_t flag, uint32_t epoch, uint64_t value) {
  return (flag << 62) | ((uint64_t)epoch << 40) | (value & ((1ull << 40) - 1));
}

// Called by one thread: publish chunk c's aggregate (or inclusive for c == 0).
__device__ __forceinline__ void lookback_publish(const LaunchCtx& ctx, uint64_t c, uint64_t agg) {
  st_relaxed_u64(ctx.status + c, make_status(c == 0 ? kFlagInc : kFlagAgg, ctx.epoch, agg));
}

// Called by a whole warp for chunk c: returns the exclusive prefix of the
// aggregates of chunks [0, c) and publishes chunk c's inclusive prefix. Lane i
// inspects chunk c−1−i of a 32-chunk window; the window moves back until an
// inclusive prefix is found. (Measured alternatives, all slower on B200 with
// scripts/ab_time.py: a 128-wide window, propagation of the resolved prefixes,
// two storer warps per CTA; the poll back-off (16 ns … 1 µs) does not matter.)
#ifndef LCF_LB_SLEEP
#define LCF_LB_SLEEP 64
#endif
// c_min: the launch's first chunk (a tile-range decode, lcf_api.cu): chunks
// below it belong to earlier launches and count as a zero inclusive prefix.
__device__ __forceinline__ uint64_t lookback_warp(const LaunchCtx& ctx, uint64_t c, uint64_t agg,
                                                  uint64_t c_min = 0) {
  const unsigned lane = threadIdx.x & 31;
  if (c == c_min) return 0;
  uint64_t excl = 0;
  int64_t pos = (int64_t)c - 1;
  while (true) {
    const int64_t idx = pos - (int64_t)lane;
    uint64_t s = 0;
    bool valid, incl;
    unsigned need, bad;
    int first_incl;
    while (true) {
      if (idx >= (int64_t)c_min) {
        s = ld_relaxed_u64(ctx.status + idx);
        const uint32_t ep = (uint32_t)(s >> 40) & 0x3FFFFFu;
        valid = (s >> 62) != 0 && ep == ctx.epoch;
        incl = valid && (s >> 62) == kFlagInc;
      } else {
        s = 0;
        valid = incl = true;
      }
      const unsigned incl_mask = __ballot_sync(0xFFFFFFFFu, incl);
      first_incl = incl_mask ? __ffs(incl_mask) - 1 : 32;
      need = first_incl == 32 ? 0xFFFFFFFFu : ((2u << first_incl) - 1u);
      bad = __ballot_sync(0xFFFFFFFFu, !valid) & need;
      if (!bad) break;
      __nanosleep(LCF_LB_SLEEP);
    }
    uint64_t v = ((int)lane <= first_incl && idx >= (int64_t)c_min) ? (s & ((1ull << 40) - 1)) : 0;
#pragma unroll
    for (int d = 16; d >= 1; d >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, d);
    excl += v;
    if (first_incl < 32) break;
    pos -= 32;
  }
  if (lane == 0) st_relaxed_u64(ctx.status + c, make_status(kFlagInc, ctx.epoch, excl + agg));
  return excl;
}

// ---- word helpers ------------------------------------------------------------
__device__ __forceinline__ int bitlen(uint32_t v) { return 32 - __clz(v); }
__device__ __forceinline__ int bitlen(uint64_t v) { return 64 - __clzll(v); }
__device__ __forceinline__ uint32_t tcms(uint32_t d) { return (d << 1) ^ (uint32_t)((int32_t)d >> 31); }
__device__ __forceinline__ uint64_t tcms(uint64_t d) {  // on 32-bit halves: one shared sign mask
  const uint32_t lo = (uint32_t)d, hi = (uint32_t)(d >> 32);
  const uint32_t m = (uint32_t)((int32_t)hi >> 31);
  return ((uint64_t)(__funnelshift_l(lo, hi, 1) ^ m) << 32) | ((lo << 1) ^ m);
}
__device__ __forceinline__ uint32_t tcms_inv(uint32_t u) { return (u >> 1) ^ (0u - (u & 1u)); }
__device__ __forceinline__ uint64_t tcms_inv(uint64_t u) {  // on 32-bit halves: one shared sign mask
  const uint32_t lo = (uint32_t)u, hi = (uint32_t)(u >> 32);
  const uint32_t m = (uint32_t)((int32_t)(lo << 31) >> 31);
  return ((uint64_t)((hi >> 1) ^ m) << 32) | (__funnelshift_r(lo, hi, 1) ^ m);
}

// 128-bit value (lo, hi) shifted left by s (0..127) / right by s.
__device__ __forceinline__ void shl128(uint64_t& lo, uint64_t& hi, unsigned s) {
  if (s == 0) return;
  if (s >= 64) { hi = lo << (s - 64); lo = 0; return; }
  hi = (hi << s) | (lo >> (64 - s));
  lo <<= s;
}
__device__ __forceinline__ void shr128(uint64_t& lo, uint64_t& hi, unsigned s) {
  if (s == 0) return;
  if (s >= 64) { lo = hi >> (s - 64); hi = 0; return; }
  lo = (lo >> s) | (hi << (64 - s));
  hi >>= s;
}
__device__ __forceinline__ uint64_t mask64(unsigned w) { return w >= 64 ? ~0ull : ((1ull << w) - 1); }

// ---- warp bit-string emission -------------------------------------------------
// Every lane holds a bit string (lo, hi: up to 128 bits, `len` bits) that goes
// to absolute bit offset `off` of a u32-word buffer `buf` in shared memory; the
// lanes' strings are consecutive and non-overlapping (lane l+1 starts where lane
// l ends). Each touched word is written exactly once, by one lane, with a plain
// store: a word shared by several lanes is OR-combined with a segmented warp
// scan. Words shared with strings emitted by OTHER warps (the warp's first and
// last word) are combined with atomicOr when `edge_atomic` is set; the caller
// then guarantees those words start zeroed.
__device__ __forceinline__ void emit_bits_warp(uint32_t* buf, uint64_t off, unsigned len,
                                               uint64_t lo, uint64_t hi, bool edge_atomic,
                                               bool long_strings = false) {
  const unsigned lane = threadIdx.x & 31;
  const uint32_t F = (uint32_t)(off >> 5);
  const unsigned r = (unsigned)(off & 31);
  // 160-bit window t0..t4 = string << r
  const uint32_t s0 = (uint32_t)lo, s1 = (uint32_t)(lo >> 32), s2 = (uint32_t)hi, s3 = (uint32_t)(hi >> 32);
  const uint32_t t0 = s0 << r, t1 = __funnelshift_l(s0, s1, r), t2 = __funnelshift_l(s1, s2, r),
                 t3 = __funnelshift_l(s2, s3, r), t4 = __funnelshift_l(s3, 0u, r);
  const unsigned nw = len ? ((r + len + 31) >> 5) : 0;  // words touched (0..5)
  const uint32_t key = nw ? F + nw - 1 : F;             // last word touched
  uint32_t last = nw <= 1 ? t0 : nw == 2 ? t1 : nw == 3 ? t2 : nw == 4 ? t3 : t4;
  if (nw == 0) last = 0;
  // segmented inclusive OR-scan of the last words, keyed by word index
  // (long_strings: the caller guarantees every string has ≥ 32 bits, so a word
  // is shared by at most two lanes and no accumulation is needed)
  uint32_t S = last;
  if (!long_strings)
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t oS = __shfl_up_sync(0xFFFFFFFFu, S, d);
    const uint32_t oK = __shfl_up_sync(0xFFFFFFFFu, key, d);
    if ((int)lane >= d && oK == key) S |= oS;
  }
  const uint32_t prevS = __shfl_up_sync(0xFFFFFFFFu, S, 1);
  const uint32_t prevK = __shfl_up_sync(0xFFFFFFFFu, key, 1);
  const uint32_t nextF = __shfl_down_sync(0xFFFFFFFFu, F, 1);
  const uint32_t firstW = __shfl_sync(0xFFFFFFFFu, F, 0);
  const uint32_t lastW = __shfl_sync(0xFFFFFFFFu, key, 31);
  auto put = [&](uint32_t idx, uint32_t v) {
    if (edge_atomic && (idx == firstW || idx == lastW)) atomicOr(buf + idx, v);
    else buf[idx] = v;
  };
  if (nw >= 2) {
    uint32_t first = t0;
    if (lane > 0 && prevK == F) first |= prevS;
    put(F, first);
    if (nw > 2) put(F + 1, t1);
    if (nw > 3) put(F + 2, t2);
    if (nw > 4) put(F + 3, t3);
  }
  // an empty string at a word boundary carries nothing: it must not write
  if ((nw >= 1 || r != 0) && (lane == 31 || nextF != key)) put(key, S);
}

}  // namespace lcf
