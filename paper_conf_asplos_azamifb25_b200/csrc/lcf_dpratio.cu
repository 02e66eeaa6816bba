// lcf_dpratio.cu — DPratio = per chunk (RARE ∘ RAZE ∘ DIFFMS₆₄) over FCM(x)
// (§3.2) on sm_100a.
//
// Compress (4 launches):
//   fcm_hash_kernel   h(i) from x[i−1..i−3] (A-13) and the index, coalesced
//   CUB radix sort    (h, i) pairs on the 20 key bits — stable, so equal hashes
//                     stay in index order (L197: "we use the CUB library")
//   fcm_match_kernel  per sorted position: the nearest of the 4 preceding pairs
//                     with the same hash and the same 64-bit word (A-14); the
//                     block stages its sorted window and the gathered words in
//                     shared memory, then scatters the 32-bit distance
//   dpratio_encode    persistent pipeline; item = 2048-word tile t → chunk 2t
//                     (V) and 2t+1 (Dist) (A-16); per chunk DIFFMS₆₄ → RAZE →
//                     RARE in shared memory (L201: histogram of leading-zero
//                     counts by warp-aggregated shared atomics; k from the prefix
//                     sums; bit fields emitted with warp segmented scans)
// Decompress (1 launch): dpratio_decode — per tile: RARE⁻¹ → RAZE⁻¹ → DIFFMS⁻¹
//   for V and Dist, then the FCM decode of the tile (L197) fused in: references
//   inside the tile are resolved by pointer jumping in shared memory, references
//   to earlier tiles read the already written output after an acquire on that
//   tile's completion flag (tiles complete in ticket order, so no cycles).

#include "lcf_persist.cuh"

namespace lcf {
namespace {

constexpr int kDW = 8;                 // compute warps
constexpr uint32_t kDT = kDW * 32;     // compute threads
#ifndef LCF_DP_OUT
#define LCF_DP_OUT 2
#endif
constexpr int kDOut = LCF_DP_OUT, kDBatch = 4;  // output slots (encode), tiles per ticket (decode)
constexpr int kDEncThreads = (2 + kDW) * 32, kDDecThreads = (1 + kDW) * 32;
constexpr uint32_t kBarD = 1;
constexpr uint32_t kTileWords = 2048;
static_assert(kDT * 8 == kTileWords, "the raw V fallback gives each compute thread 8 words");

__device__ __forceinline__ void bar_d() { named_bar_sync(kBarD, kDT); }
__device__ __forceinline__ bool bar_d_or(bool p) {
  uint32_t r;
  asm volatile("{\n .reg .pred pi, po;\n setp.ne.u32 pi, %1, 0;\n bar.red.or.pred po, %2, %3, pi;\n selp.u32 %0, 1, 0, po;\n}"
               : "=r"(r)
               : "r"((uint32_t)p), "r"(kBarD), "r"(kDT)
               : "memory");
  return r != 0;
}

// ============================ RAZE / RARE in shared memory ============================
// clz histogram: plain shared atomics (1, measured fastest: the hardware
// serialises equal bins within a warp cheaply) or match-aggregated ones (0)
#ifndef LCF_HIST_MODE
#define LCF_HIST_MODE 1
#endif
struct AdaptScratch {
  uint32_t hist[65];
  uint32_t cnt[64];     // per (round, warp) set counts → exclusive prefix
  uint32_t b1[64];      // B1 bitmap words (n ≤ 2048 bits)
  uint32_t c1m[32], off1[32], b2[32];  // encoder plan → emit: warp 0's B2 bits, nr(B1) offsets
  uint32_t k, flag, s1, s2, nr1, b3;
  uint32_t wtot[kDW];                   // encoder: set words per warp
  uint16_t rank0[kDT];                  // encoder: set words before thread t's 8 words
};

__device__ __forceinline__ uint32_t clz64(uint64_t v) { return __clzll(v); }

// 64-bit field of width w (≤ 64) at bit position P of the little-endian word
// stream at `base` (4-byte aligned; reads up to 12 bytes).
__device__ __forceinline__ uint64_t get_field(const uint32_t* base, uint64_t P, uint32_t w) {
  if (w == 0) return 0;
  const uint32_t* p = base + (P >> 5);
  const uint32_t r = P & 31;
  const uint32_t lo = __funnelshift_r(p[0], p[1], r), hi = __funnelshift_r(p[1], p[2], r);
  const uint64_t v = ((uint64_t)hi << 32) | lo;
  return w >= 64 ? v : v & ((1ull << w) - 1);
}

// Words 8·tid … 8·tid+7 of sv with 16-byte shared loads; quad q of thread t is
// read in slot q ^ ((t >> 1) & 3), which spreads the eight threads of a
// wavefront over distinct banks. Words at or past n are returned as 0. sv must
// be 16-byte aligned with readable slack up to word 8·kDT.
#ifndef LCF_LOAD8_SWZ
#define LCF_LOAD8_SWZ 0
#endif
__device__ __forceinline__ void load8(const uint64_t* sv, uint32_t n, uint32_t tid, uint64_t (&v)[8]) {
  if (!LCF_LOAD8_SWZ) {  // plain 16-byte loads (4-way bank conflicts per quarter warp)
#pragma unroll
    for (uint32_t q = 0; q < 4; ++q) {
      const ulonglong2 x = reinterpret_cast<const ulonglong2*>(sv)[4 * tid + q];
      v[2 * q] = 8 * tid + 2 * q < n ? x.x : 0ull;
      v[2 * q + 1] = 8 * tid + 2 * q + 1 < n ? x.y : 0ull;
    }
    return;
  }
  const uint32_t s = (tid >> 1) & 3;
  ulonglong2 ld[4];
#pragma unroll
  for (uint32_t q = 0; q < 4; ++q) ld[q] = reinterpret_cast<const ulonglong2*>(sv)[4 * tid + (q ^ s)];
#pragma unroll
  for (uint32_t q = 0; q < 4; ++q) {
    const ulonglong2 x = s == 0 ? ld[q] : s == 1 ? ld[q ^ 1] : s == 2 ? ld[q ^ 2] : ld[q ^ 3];
    v[2 * q] = 8 * tid + 2 * q < n ? x.x : 0ull;
    v[2 * q + 1] = 8 * tid + 2 * q + 1 < n ? x.y : 0ull;
  }
}

// LSB-first bit writer for one thread's contiguous run of fields in a u32
// buffer. The run's first and last words may be shared with the neighbouring
// runs (atomicOr into a zeroed buffer); the words in between belong to this
// thread alone (plain stores).
struct BitWriter {
  uint32_t* buf;
  uint32_t widx, nb;  // current word, pending bits in acc (< 32 between puts)
  uint64_t acc;
  bool first;
  __device__ __forceinline__ BitWriter(uint32_t* b, uint64_t off)
      : buf(b), widx((uint32_t)(off >> 5)), nb((uint32_t)(off & 31)), acc(0), first(true) {}
  __device__ __forceinline__ void emit(uint32_t w) {
    if (first) atomicOr(buf + widx, w);
    else buf[widx] = w;
    first = false;
    ++widx;
  }
  // append the low w bits of f (f < 2^w, 1 ≤ w ≤ 64)
  __device__ __forceinline__ void put(uint64_t f, uint32_t w) {
    const uint64_t carry = nb ? f >> (64 - nb) : 0ull;  // bits beyond the 64-bit accumulator
    acc |= f << nb;
    nb += w;
    if (nb >= 32) {
      emit((uint32_t)acc);
      acc = (acc >> 32) | (carry << 32);
      nb -= 32;
      if (nb >= 32) {
        emit((uint32_t)acc);
        acc >>= 32;
        nb -= 32;
      }
    }
  }
  __device__ __forceinline__ void finish() {
    if (nb) atomicOr(buf + widx, (uint32_t)acc);
  }
};

// Encode L bytes at src (16-byte aligned, zero-safe slack to 16 KiB) with RAZE
// (rare = false, L189) or RARE (rare = true, L195) into dst (16-byte aligned,
// ≥ L + 3 + 32 bytes). All kDT compute threads call it; returns the output
// length (FORMAT.md §6.2–6.3). Thread t owns words 8t … 8t+7 (n ≤ 2048): its
// B1 bits are B1 byte t, and its HI and LO fields are contiguous bit runs.
__device__ __noinline__ uint32_t adaptive_plan(const uint8_t* src, uint32_t L, bool rare, AdaptScratch& sc,
                                               uint32_t tid) {
  const uint32_t warp = tid >> 5, lane = tid & 31;
  const uint32_t n = L / 8, tl = L % 8;
  const uint64_t* sv = reinterpret_cast<const uint64_t*>(src);
  // (the input was completed before a barrier of the caller; sc.hist is zero:
  // zeroed at kernel start and again by warp 0 right after reading it)
  uint64_t v[8];
  load8(sv, n, tid, v);
  const uint32_t i0 = 8 * tid;
  const uint64_t p = (rare && i0 >= 1 && i0 - 1 < n) ? sv[i0 - 1] : 0ull;  // RARE reference of word i0
  // ---- histogram of clz(v_i ⊕ ref_i) ----
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    const uint64_t ref = rare ? (j ? v[j - 1] : p) : 0ull;
    const uint32_t z = i0 + j < n ? clz64(v[j] ^ ref) : 65u;
    if (LCF_HIST_MODE == 0) {
      const uint32_t peers = __match_any_sync(0xFFFFFFFFu, z);
      if (z <= 64 && lane == (uint32_t)(__ffs(peers) - 1)) atomicAdd(&sc.hist[z], (uint32_t)__popc(peers));
    } else {
      if (z <= 64) atomicAdd(&sc.hist[z], 1u);
    }
  }
  bar_d();
  // ---- k* = smallest argmin of est(k) = k·nz(k) + (64−k)·n, k ∈ 1..64 (A-17, A-18) ----
  if (warp == 0) {
    const uint32_t c0 = sc.hist[2 * lane], c1 = sc.hist[2 * lane + 1];
    sc.hist[2 * lane] = 0;  // ready for the next plan (its atomics follow several barriers)
    sc.hist[2 * lane + 1] = 0;
    if (lane == 0) sc.hist[64] = 0;
    uint32_t s = c0 + c1;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, s, d);
      if ((int)lane >= d) s += y;
    }
    const uint32_t before = s - c0 - c1;
    const uint32_t kA = 2 * lane + 1, kB = 2 * lane + 2;  // nz(kA) = before + c0, nz(kB) = s
    const uint32_t eA = kA * (before + c0) + (64 - kA) * n, eB = kB * s + (64 - kB) * n;
    const uint32_t keyA = (eA << 7) | kA, keyB = (eB << 7) | kB;
    const uint32_t best = __reduce_min_sync(0xFFFFFFFFu, keyA < keyB ? keyA : keyB);
    if (lane == 0) sc.k = best & 127;
  }
  bar_d();
  const uint32_t k = sc.k;
  const uint32_t sh = 64 - k;  // top(v) = v >> sh (k = 64: sh = 0)
  // ---- B1 byte t = this thread's set bits; ranks of the set words ----
  uint32_t byte = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    const uint64_t ref = rare ? (j ? v[j - 1] : p) : 0ull;
    if (i0 + j < n && (v[j] >> sh) != (ref >> sh)) byte |= 1u << j;
  }
  reinterpret_cast<uint8_t*>(sc.b1)[tid] = (uint8_t)byte;
  const uint32_t c = __popc(byte);
  uint32_t x = c;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
    if ((int)lane >= d) x += y;
  }
  if (lane == 31) sc.wtot[warp] = x;
  bar_d();
  {
    uint32_t base = 0;
#pragma unroll
    for (uint32_t w = 0; w < kDW; ++w)
      if (w < warp) base += sc.wtot[w];
    sc.rank0[tid] = (uint16_t)(base + x - c);
  }
  uint32_t nr1 = 0, b2 = 0, b3 = 0, c1m = 0, off1 = 0, b1w0 = 0, b1w1 = 0;
  const uint32_t L1 = (n + 7) / 8, L2 = (L1 + 7) / 8, L3 = (L2 + 7) / 8;
  if (warp == 0) {
    uint32_t nset = 0;
#pragma unroll
    for (uint32_t w = 0; w < kDW; ++w) nset += sc.wtot[w];
    // B1 → B2 (lane: B1 bytes [8·lane, 8·lane+8) = words 2·lane, 2·lane+1)
    b1w0 = sc.b1[2 * lane];
    b1w1 = sc.b1[2 * lane + 1];
    const uint32_t prevb = __shfl_up_sync(0xFFFFFFFFu, b1w1 >> 24, 1);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const uint32_t cur = ((j < 4 ? b1w0 : b1w1) >> (8 * (j & 3))) & 0xFF;
      const uint32_t pre = j ? (((j - 1) < 4 ? b1w0 : b1w1) >> (8 * ((j - 1) & 3))) & 0xFF : (lane ? prevb : 0u);
      if (cur != pre && 8 * lane + j < L1) c1m |= 1u << j;
    }
    b2 = c1m;  // B2 byte `lane`
    uint32_t y = __popc(c1m);
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(0xFFFFFFFFu, y, d);
      if ((int)lane >= d) y += o;
    }
    off1 = y - __popc(c1m);
    nr1 = __shfl_sync(0xFFFFFFFFu, y, 31);
    const uint32_t pb2 = __shfl_up_sync(0xFFFFFFFFu, b2, 1);
    b3 = __ballot_sync(0xFFFFFFFFu, lane < L2 && b2 != (lane ? pb2 : 0u));
    const uint32_t nr2 = __popc(b3);
    const uint32_t hib = (nset * k + 7) / 8, lob = (n * (64 - k) + 7) / 8;
    const uint32_t total = 3 + hib + lob + tl + nr1 + nr2 + L3;
    if (lane == 0) {
      sc.flag = total >= 3 + L;  // bypass (A-23)
      sc.s1 = total;
      sc.s2 = hib;
      sc.nr1 = nr1;
      sc.b3 = b3;
    }
    sc.c1m[lane] = c1m;
    sc.off1[lane] = off1;
    sc.b2[lane] = b2;
  }
  bar_d();
  return sc.flag ? 3 + L : sc.s1;
}

// Second half of RAZE/RARE: writes the planned output (adaptive_plan must have
// run on the same input just before).
__device__ __noinline__ void adaptive_emit(const uint8_t* src, uint32_t L, uint8_t* dst, bool rare,
                                           AdaptScratch& sc, uint32_t tid) {
  const uint32_t warp = tid >> 5, lane = tid & 31;
  const uint32_t n = L / 8, tl = L % 8;
  const uint64_t* sv = reinterpret_cast<const uint64_t*>(src);
  const uint32_t k = sc.k, sh = 64 - k;
  const uint32_t L1 = (n + 7) / 8, L2 = (L1 + 7) / 8, L3 = (L2 + 7) / 8;
  (void)L1;
  (void)L2;
  (void)rare;
  const bool bypass = sc.flag;
  const uint32_t total = sc.s1, hib = sc.s2, nr1 = sc.nr1, b3 = sc.b3;
  if (bypass) {  // dst[3 + j] = src[j], one funnel shift per output word
    const uint32_t* sw = reinterpret_cast<const uint32_t*>(src);
    uint32_t* dw = reinterpret_cast<uint32_t*>(dst);
    const uint32_t nw = (L + 3 + 3) / 4;
    for (uint32_t w = tid; w < nw; w += kDT) {
      const uint32_t lo = w ? sw[w - 1] : 0u;
      const uint32_t hi = 4 * w < L ? sw[w] : 0u;
      uint32_t val = w ? __funnelshift_r(lo, hi, 8) : ((L & 0xFFFFu) | (hi << 24));
      const uint32_t keep = 3 + L - 4 * w;  // bytes of this word inside the output
      if (keep < 4) val &= (1u << (8 * keep)) - 1u;
      dw[w] = val;
    }
    bar_d();
    return;
  }
  uint32_t* dw = reinterpret_cast<uint32_t*>(dst);
  for (uint32_t j = tid; j < (total + 7) / 4 + 1; j += kDT) dw[j] = 0;
  uint64_t v[8];
  load8(sv, n, tid, v);
  const uint32_t i0 = 8 * tid;
  const uint32_t byte = reinterpret_cast<const uint8_t*>(sc.b1)[tid];
  const uint32_t rank0 = sc.rank0[tid];
  bar_d();
  // ---- HI: top fields of the set words (rank order), LO: low fields of all words ----
  const uint64_t hi_base = 24, lo_base = 8ull * (3 + hib);
  const uint32_t wl = 64 - k;
  const uint64_t lmask = wl >= 64 ? ~0ull : ((1ull << wl) - 1);
  if (byte) {
    BitWriter bw(dw, hi_base + (uint64_t)rank0 * k);
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if ((byte >> j) & 1) bw.put(v[j] >> sh, k);
    bw.finish();
  }
  if (wl && i0 < n) {
    BitWriter bw(dw, lo_base + (uint64_t)i0 * wl);
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (i0 + j < n) bw.put(v[j] & lmask, wl);
    bw.finish();
  }
  // ---- header, tail bytes, nr(B1), nr(B2), B3: byte ORs into the zeroed
  // words, concurrent with the bit writers (whose edge words they may share) ----
  auto put_byte = [&](uint32_t pos, uint32_t val) {
    atomicOr(dw + (pos >> 2), (val & 0xFFu) << (8 * (pos & 3)));
  };
  const uint32_t after = 3 + hib + (n * wl + 7) / 8;
  if (tid == 0) atomicOr(dw, (L & 0xFFFFu) | (k << 16));
  if (tid < tl) put_byte(after + tid, src[8 * n + tid]);
  if (warp == 0) {
    const uint32_t c1m = sc.c1m[lane], b2 = sc.b2[lane];
    const uint32_t b1w0 = sc.b1[2 * lane], b1w1 = sc.b1[2 * lane + 1];
    uint32_t p = after + tl + sc.off1[lane];
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if ((c1m >> j) & 1) put_byte(p++, (j < 4 ? b1w0 : b1w1) >> (8 * (j & 3)));
    if ((b3 >> lane) & 1) put_byte(after + tl + nr1 + __popc(b3 & ((1u << lane) - 1)), b2);
    if (lane < L3) put_byte(total - L3 + lane, b3 >> (8 * lane));
  }
  bar_d();
}

__device__ __forceinline__ uint32_t adaptive_encode(const uint8_t* src, uint32_t L, uint8_t* dst, bool rare,
                                                    AdaptScratch& sc, uint32_t tid) {
  const uint32_t len = adaptive_plan(src, L, rare, sc, tid);
  adaptive_emit(src, L, dst, rare, sc, tid);
  return len;
}

// Decode a RAZE/RARE stream of `len` bytes at src (16-byte aligned, ≥ 16 bytes
// of readable slack) into dst (8-byte aligned, capacity cap). Returns the
// decoded length or −1 if malformed. All kDT compute threads call it.
__device__ int adaptive_decode(const uint8_t* src, uint32_t len, uint8_t* dst, uint32_t cap, bool rare,
                               AdaptScratch& sc, uint32_t tid) {
  const uint32_t warp = tid >> 5, lane = tid & 31;
  if (len < 3) return -1;
  const uint32_t L = src[0] | ((uint32_t)src[1] << 8), k = src[2];
  if (L > cap) return -1;
  if (k == 0) {  // bypass: dst[j] = src[3 + j], one funnel shift per word
    if (len != 3 + L) return -1;
    const uint32_t* sw = reinterpret_cast<const uint32_t*>(src);
    uint32_t* dw = reinterpret_cast<uint32_t*>(dst);
    for (uint32_t w = tid; w < (L + 3) / 4; w += kDT) dw[w] = __funnelshift_r(sw[w], sw[w + 1], 24);
    bar_d();
    return (int)L;
  }
  if (k > 64) return -1;
  const uint32_t n = L / 8, tl = L % 8, L1 = (n + 7) / 8, L2 = (L1 + 7) / 8, L3 = (L2 + 7) / 8;
  const uint32_t wl = 64 - k;
  if (warp == 0) {
    int bad = len < 3 + L3;
    uint32_t b3 = 0;
    if (!bad)
      for (uint32_t j = 0; j < L3; ++j) b3 |= (uint32_t)src[len - L3 + j] << (8 * j);
    const uint32_t v2 = L2 >= 32 ? 0xFFFFFFFFu : ((1u << L2) - 1u);
    const int32_t s2 = (int32_t)len - (int32_t)L3 - __popc(b3 & v2);
    if (s2 < 3) bad = 1;
    const uint32_t r2 = __popc(b3 & v2 & (0xFFFFFFFFu >> (31 - lane)));
    const uint32_t b2 = (!bad && lane < L2 && r2) ? src[s2 + r2 - 1] : 0u;  // B2 byte `lane`
    // B1 bytes [8·lane, 8·lane+8) from the bits of B2 byte `lane`
    const uint32_t vb = (8 * lane >= L1) ? 0u : (L1 - 8 * lane >= 8 ? 0xFFu : ((1u << (L1 - 8 * lane)) - 1u));
    const uint32_t bits = b2 & vb;
    uint32_t x = __popc(bits);
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
      if ((int)lane >= d) x += y;
    }
    const int32_t s1 = s2 - (int32_t)__shfl_sync(0xFFFFFFFFu, x, 31);
    if (s1 < 3) bad = 1;
    bad = __any_sync(0xFFFFFFFFu, bad);
    uint32_t r = x - __popc(bits), w0 = 0, w1 = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      r += (bits >> j) & 1;
      const uint32_t val = (!bad && r) ? src[s1 + r - 1] : 0u;
      if (j < 4) w0 |= val << (8 * j);
      else w1 |= val << (8 * (j - 4));
    }
    // B1 words cover bits 64·lane .. : mask bits ≥ n
    const uint32_t nb0 = n > 64 * lane ? n - 64 * lane : 0;
    if (nb0 < 32) w0 &= nb0 ? ((1u << nb0) - 1u) : 0u;
    if (nb0 < 64) w1 &= nb0 > 32 ? ((1u << (nb0 - 32)) - 1u) : 0u;
    sc.b1[2 * lane] = w0;
    sc.b1[2 * lane + 1] = w1;
    const uint32_t cw0 = __popc(w0), cw1 = __popc(w1);
    uint32_t c = cw0 + cw1;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, c, d);
      if ((int)lane >= d) c += y;
    }
    sc.cnt[2 * lane] = c - cw0 - cw1;
    sc.cnt[2 * lane + 1] = c - cw1;
    const uint32_t nset = __shfl_sync(0xFFFFFFFFu, c, 31);
    const uint32_t hib = (nset * k + 7) / 8, lob = (n * wl + 7) / 8;
    if (!bad && (int32_t)(3 + hib + lob + tl) != s1) bad = 1;
    if (lane == 0) {
      sc.flag = bad;
      sc.s2 = hib;
    }
  }
  bar_d();
  if (sc.flag) return -1;
  const uint32_t hib = sc.s2;
  const uint32_t* sw = reinterpret_cast<const uint32_t*>(src);
  const uint64_t lo_base = 8ull * (3 + hib);
  // word i = 32·(b1 word index) + lane: B1 word q = 8r + warp covers i = 256 r + 32 warp + lane
#pragma unroll
  for (int r = 0; r < 8; ++r) {
    const uint32_t i = tid + kDT * r;
    const uint32_t q = r * kDW + warp;
    const uint32_t bw = sc.b1[q];
    const uint32_t re = sc.cnt[q] + __popc(bw & ((1u << lane) - 1));  // set words before i
    const bool set = (bw >> lane) & 1;
    if (i < n) {
      uint64_t tp;
      if (rare) {
        const uint32_t ri = re + set;  // set words up to and including i
        tp = ri ? get_field(sw, 24 + (uint64_t)(ri - 1) * k, k) : 0;
      } else {
        tp = set ? get_field(sw, 24 + (uint64_t)re * k, k) : 0;
      }
      const uint64_t lw = get_field(sw, lo_base + (uint64_t)i * wl, wl);
      *reinterpret_cast<uint64_t*>(dst + 8 * i) = k == 64 ? tp : ((tp << wl) | lw);
    }
  }
  if (tid < tl) dst[8 * n + tid] = src[lo_base / 8 + (n * wl + 7) / 8 + tid];
  bar_d();
  return (int)L;
}

// CTA-wide exclusive scan of u64 over the kDT compute threads (slot `sh`).
__device__ __forceinline__ uint64_t cta_scan_u64(uint64_t v, uint64_t* sh, uint32_t tid, uint64_t& total) {
  const uint32_t warp = tid >> 5, lane = tid & 31;
  uint64_t x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint64_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
    if ((int)lane >= d) x += y;
  }
  if (lane == 31) sh[warp] = x;
  bar_d();
  uint64_t base = 0;
  total = 0;
#pragma unroll
  for (uint32_t i = 0; i < kDW; ++i) {
    const uint64_t s = sh[i];
    if (i < warp) base += s;
    total += s;
  }
  bar_d();  // the slot may be reused right away
  return base + x - v;
}

// =================================== encode ======================================
struct DEncSmem {
  alignas(128) uint64_t xin[kTileWords];        // stage: x tile
  alignas(128) uint32_t din[kTileWords];        // stage: FCM distances of the tile
  alignas(128) uint32_t dcp[kTileWords];        // copy of din: the stage is released after V's DIFFMS
  alignas(128) uint64_t w[kTileWords + 8];      // DIFFMS words of V or Dist
  alignas(128) uint8_t rz[kChunkBytes + 128];   // RAZE output
  alignas(128) uint32_t out[kDOut][(kChunkBytes + 128) / 4];
  uint64_t full_in[1], empty_in[1], full_out[kDOut], empty_out[kDOut];
  uint64_t in_chunk[1], out_chunk[kDOut];
  uint32_t out_len[kDOut], out_raw[kDOut];
  uint64_t scan[kDW];
  alignas(16) uint8_t zc[64];  // the Dist chunk of a full tile without distances: its stream, once made
  uint32_t zlen;               // (0 = not yet)
  AdaptScratch sc;
};

__device__ __forceinline__ void d_enc_loader(DEncSmem& S, const EncArgs& a, const LaunchCtx& ctx, uint32_t lane) {
  const uint64_t T = a.n_chunks / 2;
  for (uint32_t it = 0;; ++it) {
    const uint32_t ph = it & 1;
    mbar_wait(&S.empty_in[0], ph ^ 1);
    uint64_t t = 0;
    if (lane == 0) t = atomicAdd(ctx.ticket, 1ull);
    t = __shfl_sync(0xFFFFFFFFu, t, 0);
    if (t >= T) {
      if (lane == 0) {
        S.in_chunk[0] = kNoChunk;
        mbar_arrive(&S.full_in[0]);
        ticket_retire(ctx);
      }
      return;
    }
    const uint32_t m = (uint32_t)umin64(kTileWords, a.n_words_total - t * kTileWords);
    if (lane == 0) {
      trace_stamp(a, 2 * t, 0);
      trace_stamp(a, 2 * t + 1, 0);
    }
    const uint64_t* xs = reinterpret_cast<const uint64_t*>(a.in) + t * kTileWords;
    const uint32_t* ds = a.fcm_dist + t * kTileWords;
    if ((m & 3) == 0) {
      if (lane == 0) {
        S.in_chunk[0] = t;
        mbar_arrive_expect_tx(&S.full_in[0], 12 * m);
        tma_load_1d(S.xin, xs, 8 * m, &S.full_in[0]);
        tma_load_1d(S.din, ds, 4 * m, &S.full_in[0]);
      }
    } else {
      for (uint32_t i = lane; i < m; i += 32) {
        S.xin[i] = xs[i];
        S.din[i] = ds[i];
      }
      if (lane == 0) S.in_chunk[0] = t;
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.full_in[0]);
    }
  }
}

__device__ __forceinline__ void d_enc_compute(DEncSmem& S, const EncArgs& a, const LaunchCtx& ctx, uint32_t tid) {
  const uint32_t warp = tid >> 5, lane = tid & 31;
  uint32_t oit = 0;  // output-slot iteration (two chunks per tile)
  for (uint32_t it = 0;; ++it) {
    mbar_wait(&S.full_in[0], it & 1);
    const uint64_t t = S.in_chunk[0];
    if (t == kNoChunk) {
      enc_forward_end<kDOut, 1>(S, oit, warp, lane);
      return;
    }
    const uint32_t m = (uint32_t)umin64(kTileWords, a.n_words_total - t * kTileWords);
    bool dist_zero = false;  // the tile has no FCM match (set by part 0)
    for (uint32_t part = 0; part < 2; ++part, ++oit) {  // chunk 2t: V, chunk 2t+1: Dist (A-16)
      const uint64_t c = 2 * t + part;
      if (tid == 0) trace_stamp(a, c, 1);
      const uint32_t o = oit % kDOut, pho = (oit / kDOut) & 1;
      const bool cacheable = part == 1 && dist_zero && m == kTileWords;
      if (cacheable && S.zlen) {  // the fixed stream of an all-zero Dist chunk, made once per CTA
        const uint32_t len = S.zlen;
        if (tid == 0) {
          lookback_publish(ctx, c, round16(len));
          trace_stamp(a, c, 2);
        }
        mbar_wait(&S.empty_out[o], pho ^ 1);
        if (tid < round16(len) / 4) S.out[o][tid] = reinterpret_cast<const uint32_t*>(S.zc)[tid];
        if (tid == 0) {
          S.out_chunk[o] = c;
          S.out_len[o] = len;
          S.out_raw[o] = 0;
          trace_stamp(a, c, 3);
        }
        fence_proxy_async_smem();
        bar_d();
        if (tid == 0) trace_stamp(a, c, 4);
        if (lane == 0) mbar_arrive(&S.full_out[o]);
        continue;
      }
      // FCM outputs (L170–185) and DIFFMS₆₄ (L187) into w[]
      uint64_t nzacc = 0;
      uint32_t dor = 0;
      for (uint32_t i = tid; i < m; i += kDT) {
        uint64_t cur, prev;
        if (part == 0) {
          const uint32_t d = S.din[i], dp = i ? S.din[i - 1] : 0u;
          cur = d ? 0ull : S.xin[i];
          prev = i ? (dp ? 0ull : S.xin[i - 1]) : 0ull;
          S.dcp[i] = d;
          dor |= d;
        } else {
          cur = S.dcp[i];
          prev = i ? (uint64_t)S.dcp[i - 1] : 0ull;
        }
        const uint64_t wv = tcms((uint64_t)(cur - prev));
        S.w[i] = wv;
        nzacc |= wv;
      }
      // RAZE then RARE (L189–201)
      uint32_t l1;
      const bool any = bar_d_or(nzacc != 0);
      if (part == 0) dist_zero = !bar_d_or(dor != 0);
      // the tile's stage has been read (V's DIFFMS words are in w, the
      // distances in dcp): hand it back so the next tile loads during this one
      if (part == 0 && lane == 0) mbar_arrive(&S.empty_in[0]);
      if (any) {
        l1 = adaptive_encode(reinterpret_cast<const uint8_t*>(S.w), 8 * m, S.rz, false, S.sc, tid);
      } else {
        // all-zero DIFFMS words (e.g. the Dist chunk of a tile without FCM
        // matches): RAZE's plan is fixed — every clz is 64, so k = 64, B1..B3
        // are zero and nothing repeats — and the stream is L | k=64 | L3 zero
        // bytes (FORMAT.md §6.2; the same bytes adaptive_encode writes)
        const uint32_t L = 8 * m, L3 = (((m + 7) / 8 + 7) / 8 + 7) / 8;
        if (tid < 3 + L3) S.rz[tid] = tid == 0 ? (uint8_t)L : tid == 1 ? (uint8_t)(L >> 8) : tid == 2 ? 64 : 0;
        l1 = 3 + L3;
        bar_d();  // adaptive_plan reads its input before its first barrier
      }
      // RARE is planned first: the chunk's size — and its aggregate for the
      // look-back of later chunks — is known before an output slot is needed
      const uint32_t l2 = adaptive_plan(S.rz, l1, true, S.sc, tid);
      const uint32_t raw_len = 8 * m;
      const bool raw = l2 >= raw_len;  // L104, ties → raw
      const uint32_t len = raw ? raw_len : l2;
      if (tid == 0) {
        lookback_publish(ctx, c, round16(len));
        trace_stamp(a, c, 2);
      }
      mbar_wait(&S.empty_out[o], pho ^ 1);
      if (tid == 0) trace_stamp(a, c, 3);
      uint8_t* ob = reinterpret_cast<uint8_t*>(S.out[o]);
      if (raw) {  // the V / Dist words themselves
        uint64_t* ow = reinterpret_cast<uint64_t*>(ob);
        if (part == 0) {  // V = DIFFMS⁻¹(w): words 8·tid .. 8·tid+7, serial run + CTA scan
          uint64_t run = 0;
#pragma unroll
          for (uint32_t j = 0; j < 8; ++j) {
            const uint32_t i = 8 * tid + j;
            if (i < m) run += tcms_inv(S.w[i]);
          }
          uint64_t all;
          uint64_t v = cta_scan_u64(run, S.scan, tid, all);
#pragma unroll
          for (uint32_t j = 0; j < 8; ++j) {
            const uint32_t i = 8 * tid + j;
            if (i < m) {
              v += tcms_inv(S.w[i]);
              ow[i] = v;
            }
          }
        } else {
          for (uint32_t i = tid; i < m; i += kDT) ow[i] = S.dcp[i];
        }
        if (tid < 2 && (m & 1)) ow[m + tid] = 0;  // round16 pad
      } else {
        adaptive_emit(S.rz, l1, ob, true, S.sc, tid);
        if (tid < 16 && len + tid < round16(len)) ob[len + tid] = 0;
        if (cacheable && round16(len) <= sizeof(S.zc)) {  // remember it (read after later barriers)
          bar_d();
          if (tid < round16(len)) S.zc[tid] = ob[tid];
          if (tid == 0) S.zlen = len;
        }
      }
      if (tid == 0) {
        S.out_chunk[o] = c;
        S.out_len[o] = len;
        S.out_raw[o] = raw;
      }
      fence_proxy_async_smem();
      bar_d();
      if (tid == 0) trace_stamp(a, c, 4);
      if (lane == 0) mbar_arrive(&S.full_out[o]);
    }
  }
}

__global__ void __launch_bounds__(kDEncThreads) dpratio_encode_kernel(EncArgs a, LaunchCtx ctx) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  DEncSmem& S = *reinterpret_cast<DEncSmem*>(smem_raw);
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (uint32_t i = threadIdx.x; i < 65; i += blockDim.x) S.sc.hist[i] = 0;  // adaptive_plan's invariant
  if (threadIdx.x == 0) S.zlen = 0;
  if (threadIdx.x == 0) {
    mbar_init(&S.full_in[0], 1);
    mbar_init(&S.empty_in[0], kDW);
    for (int i = 0; i < kDOut; ++i) {
      mbar_init(&S.full_out[i], kDW);
      mbar_init(&S.empty_out[i], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == 0) d_enc_loader(S, a, ctx, lane);
  else if (warp == 1) enc_storer<kDOut, 1>(S, a, ctx, lane, 0);
  else d_enc_compute(S, a, ctx, threadIdx.x - 64);
}

// =================================== decode ======================================
struct DDecSmem {
  alignas(128) uint8_t in[2][kChunkBytes + 128];  // stage: V and Dist payloads of a tile
  alignas(128) uint8_t rz[2][kChunkBytes + 128];  // RARE⁻¹ outputs (RAZE streams) of V and Dist
  alignas(128) uint64_t V[kTileWords + 8];        // V, then the decoded tile in place
  alignas(128) uint64_t D[kTileWords + 8];
  int32_t pj[2][kDT];                             // pointer jumping: target (−1 done)
  uint64_t vj[2][kDT];
  uint64_t full_in[1], empty_in[1];
  uint64_t tile[1];
  uint32_t len[1][2], flags[1];
  uint64_t scan[kDW];
  AdaptScratch sc;
  int32_t bad;
};

__device__ __forceinline__ void d_dec_loader(DDecSmem& S, const DecArgs& a, const LaunchCtx& ctx, uint32_t lane) {
  uint64_t n_words = 0, n_chunks = 0, base = 0, payload = 0;
  const bool hdr_ok = read_header(a, ctx, n_words, n_chunks, base, payload);
  const bool small = hdr_ok && n_words * 8 > a.out_capacity;
  const uint64_t T = n_chunks / 2;
  uint32_t it = 0;
  for (;;) {
    uint64_t tb = 0;
    if (lane == 0) tb = atomicAdd(ctx.ticket, 1ull);
    tb = __shfl_sync(0xFFFFFFFFu, tb, 0) * kDBatch;
    if (!hdr_ok || small || tb >= T) {
      mbar_wait(&S.empty_in[0], (it & 1) ^ 1);
      if (lane == 0) {
        if (tb == 0 && !hdr_ok) record_error(ctx, DERR_CORRUPT);
        if (tb == 0 && small) record_error(ctx, DERR_SMALL);
        S.tile[0] = kNoChunk;
        mbar_arrive(&S.full_in[0]);
        ticket_retire(ctx);
      }
      return;
    }
    const uint32_t nb = (uint32_t)umin64(kDBatch, T - tb);  // tiles; chunks 2tb .. 2tb + 2nb − 1
    const uint64_t c = 2 * tb + lane;
    uint32_t len = 0, raw = 0;
    bool bad = false;
    if (lane < 2 * nb) {
      const uint32_t e = reinterpret_cast<const uint32_t*>(a.stream + kHeaderBytes)[c];
      len = e & ~kRawFlag;
      raw = e >> 31;
      const uint32_t m = (uint32_t)umin64(kTileWords, n_words - (c / 2) * kTileWords);
      bad = raw ? len != 8 * m : len >= 8 * m;
      lookback_publish(ctx, c, bad ? 0 : round16(len));
    }
    const uint64_t agg = (lane < 2 * nb && !bad) ? round16(len) : 0;
    uint64_t x = agg;
#pragma unroll
    for (int d = 1; d < 2 * kDBatch; d <<= 1) {
      const uint64_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
      if ((int)lane >= d) x += y;
    }
    x -= agg;
    const uint64_t base_b = lookback_warp(ctx, 2 * tb, __shfl_sync(0xFFFFFFFFu, agg, 0));
    const uint64_t excl = base_b + x;
    if (lane > 0 && lane < 2 * nb) st_relaxed_u64(ctx.status + c, make_status(kFlagInc, ctx.epoch, excl + agg));
    const uint64_t end = excl + round16(len);
    if (lane < 2 * nb && !bad && (end > payload || (c == n_chunks - 1 && end != payload))) bad = true;
    for (uint32_t j = 0; j < nb; ++j, ++it) {
      const uint32_t l0 = __shfl_sync(0xFFFFFFFFu, len, 2 * j), l1 = __shfl_sync(0xFFFFFFFFu, len, 2 * j + 1);
      const uint32_t r0 = __shfl_sync(0xFFFFFFFFu, raw, 2 * j), r1 = __shfl_sync(0xFFFFFFFFu, raw, 2 * j + 1);
      const bool b0 = __shfl_sync(0xFFFFFFFFu, bad, 2 * j), b1 = __shfl_sync(0xFFFFFFFFu, bad, 2 * j + 1);
      const uint64_t e0 = __shfl_sync(0xFFFFFFFFu, excl, 2 * j), e1 = __shfl_sync(0xFFFFFFFFu, excl, 2 * j + 1);
      if (lane == 0) trace_stamp(a, tb + j, 0);
      mbar_wait(&S.empty_in[0], (it & 1) ^ 1);
      if (lane == 0) {
        trace_stamp(a, tb + j, 1);
        const bool bb = b0 || b1;
        if (bb) record_error(ctx, DERR_CORRUPT);
        S.tile[0] = tb + j;
        S.len[0][0] = l0;
        S.len[0][1] = l1;
        S.flags[0] = r0 | (r1 << 1) | (bb ? 4u : 0u);
        const uint32_t tx = bb ? 0 : (uint32_t)(round16(l0) + round16(l1));
        if (tx) {
          mbar_arrive_expect_tx(&S.full_in[0], tx);
          if (l0) tma_load_1d(S.in[0], a.stream + base + e0, (uint32_t)round16(l0), &S.full_in[0]);
          if (l1) tma_load_1d(S.in[1], a.stream + base + e1, (uint32_t)round16(l1), &S.full_in[0]);
        } else {
          mbar_arrive(&S.full_in[0]);
        }
      }
    }
  }
}

// One chunk of a tile in two steps, so that the tile's payload stage can be
// released between them. Step 1 reads the payload: RARE⁻¹ into rz (returns its
// length), or a raw chunk straight into arr (returns kRawDone; *nz = any
// non-zero word). Step 2: RAZE⁻¹ into arr and DIFFMS⁻¹ in place (*nz = any
// non-zero result). Both return −1 / false if malformed.
constexpr int kRawDone = -2;
__device__ __forceinline__ int d_decode_step1(DDecSmem& S, const uint8_t* pay, uint32_t len, bool raw, uint32_t m,
                                              uint8_t* rz, uint64_t* arr, bool& nz, uint32_t tid) {
  if (raw) {
    uint64_t acc = 0;
    for (uint32_t i = tid; i < m; i += kDT) {
      const uint64_t w = reinterpret_cast<const uint64_t*>(pay)[i];
      arr[i] = w;
      acc |= w;
    }
    nz = bar_d_or(acc != 0);
    return kRawDone;
  }
  return adaptive_decode(pay, len, rz, kChunkBytes + 3, true, S.sc, tid);
}
__device__ __forceinline__ bool d_decode_step2(DDecSmem& S, int l1, const uint8_t* rz, uint32_t m, uint64_t* arr,
                                               bool& nz, bool want_zeros, uint32_t tid) {
  if (l1 == kRawDone) return true;
  if (l1 < 0) return false;
  {  // the RAZE stream of an all-zero chunk: k = 64 and nothing but the B3
     // bytes, which a valid stream then has all zero (any set B3 bit would
     // claim nr(B2) bytes that are not there) — the encoder's fixed stream
    const uint32_t L = rz[0] | ((uint32_t)rz[1] << 8), n = L / 8;
    const uint32_t L3 = (((n + 7) / 8 + 7) / 8 + 7) / 8;
    if (l1 >= 3 && rz[2] == 64 && L == 8 * m && (uint32_t)l1 == 3 + L3) {
      bool z = true;
      for (uint32_t j = 0; j < L3; ++j) z = z && rz[3 + j] == 0;
      if (!z) return false;
      if (want_zeros)
        for (uint32_t i = tid; i < m; i += kDT) arr[i] = 0;  // DIFFMS⁻¹ of zeros
      nz = false;
      bar_d();
      return true;
    }
  }
  const int l0 = adaptive_decode(rz, (uint32_t)l1, reinterpret_cast<uint8_t*>(arr), 8 * m, false, S.sc, tid);
  if (l0 != (int)(8 * m)) return false;
  // DIFFMS⁻¹: thread owns words [8·tid, 8·tid+8), moved as 16-byte pairs
  uint64_t v[8], run = 0;
#pragma unroll
  for (int j = 0; j < 8; j += 2) {
    const ulonglong2 q = reinterpret_cast<const ulonglong2*>(arr)[4 * tid + j / 2];
    v[j] = 8 * tid + j < m ? tcms_inv((uint64_t)q.x) : 0;
    v[j + 1] = 8 * tid + j + 1 < m ? tcms_inv((uint64_t)q.y) : 0;
    run += v[j] + v[j + 1];
  }
  uint64_t tot;
  uint64_t acc = cta_scan_u64(run, S.scan, tid, tot);
  uint64_t any = 0;
#pragma unroll
  for (int j = 0; j < 8; j += 2) {
    const uint64_t a0 = acc + v[j], a1 = a0 + v[j + 1];
    acc = a1;
    reinterpret_cast<ulonglong2*>(arr)[4 * tid + j / 2] = make_ulonglong2(a0, a1);  // words ≥ m: scratch
    if (8 * tid + j < m) any |= a0;
    if (8 * tid + j + 1 < m) any |= a1;
  }
  nz = bar_d_or(any != 0);
  return true;
}

__device__ __forceinline__ void d_dec_compute(DDecSmem& S, const DecArgs& a, const LaunchCtx& ctx, uint32_t tid) {
  const uint32_t lane = tid & 31;
  const uint4 h0 = reinterpret_cast<const uint4*>(a.stream)[0];
  const uint64_t n_words = (((uint64_t)h0.w << 32) | h0.z) / 8;
  uint64_t* out = reinterpret_cast<uint64_t*>(a.out);
  // The decoded tile leaves S.V by a TMA bulk store issued by thread 0; its
  // completion (and the tile's flag) is awaited only before S.V is written
  // again, or at exit.
  uint64_t pending = kNoChunk;
  auto finish_pending = [&]() {
    if (tid == 0 && pending != kNoChunk) {
      tma_store_wait_all0();
      __threadfence();
      st_release_u32(a.tile_flag + pending, ctx.epoch);
      trace_stamp(a, pending, 7);
    }
    pending = kNoChunk;
  };
  for (uint32_t it = 0;; ++it) {
    mbar_wait(&S.full_in[0], it & 1);
    const uint64_t t = S.tile[0];
    if (t == kNoChunk) {
      finish_pending();
      return;
    }
    const uint32_t fl = S.flags[0];
    const uint32_t m = (uint32_t)umin64(kTileWords, n_words - t * kTileWords);
    if (tid == 0) trace_stamp(a, t, 2);
    bool ok = !(fl & 4), nzV = false, nzD = false;
    int l1V = -1, l1D = -1;
    if (fl & 1) {  // a raw V chunk is copied into S.V right away
      finish_pending();
      bar_d();
    }
    if (ok) {
      l1V = d_decode_step1(S, S.in[0], S.len[0][0], fl & 1, m, S.rz[0], S.V, nzV, tid);
      l1D = d_decode_step1(S, S.in[1], S.len[0][1], (fl >> 1) & 1, m, S.rz[1], S.D, nzD, tid);
    }
    // both payloads have been read (RARE⁻¹ outputs in rz, raw chunks in V / D):
    // the loader may fetch the next tile while this one finishes
    __syncwarp();
    if (lane == 0) mbar_arrive(&S.empty_in[0]);
    if (tid == 0) trace_stamp(a, t, 3);
    finish_pending();  // (step 2 writes S.V only after its first barrier)
    if (ok) ok = d_decode_step2(S, l1V, S.rz[0], m, S.V, nzV, true, tid);
    if (tid == 0) trace_stamp(a, t, 4);
    if (ok) ok = d_decode_step2(S, l1D, S.rz[1], m, S.D, nzD, false, tid);  // (D unread if all zero)
    if (tid == 0) trace_stamp(a, t, 5);
    // ---- FCM decode of the tile (L197): x[i] = Dist[i] ? x[i − Dist[i]] : V[i] ----
    const uint64_t t0 = t * kTileWords;
    bool bad = !ok;
    if (ok && nzD) {  // (no distances: x = V as it stands)
      for (uint32_t b = 0; b < m; b += kDT) {  // 256-element blocks in index order
        const uint32_t li = b + tid;
        int32_t p = -1;
        uint64_t val = 0;
        if (li < m) {
          const uint64_t d = S.D[li], gi = t0 + li;
          if (d == 0) {
            val = S.V[li];
          } else if (d > gi || S.V[li] != 0) {
            bad = true;
          } else if (gi - d >= t0 + b) {
            p = (int32_t)(gi - d - t0 - b);  // inside this block: resolve below
          } else if (gi - d >= t0) {
            val = S.V[gi - d - t0];  // earlier block of this tile: already final
          } else {  // earlier tile: wait for its completion flag, then read the output
            const uint64_t j = gi - d, tj = j / kTileWords;
            while (ld_acquire_u32(a.tile_flag + tj) != ctx.epoch) __nanosleep(100);
            val = ld_cg_u64(out + j);
          }
        }
        // pointer jumping inside the block (≤ 8 rounds; chains point backwards)
        uint32_t par = 0;
        S.pj[0][tid] = p;
        S.vj[0][tid] = val;
        while (bar_d_or(p >= 0)) {
          if (p >= 0) {
            const int32_t q = S.pj[par][p];
            if (q < 0) {
              val = S.vj[par][p];
              p = -1;
            } else {
              p = q;
            }
          }
          S.pj[par ^ 1][tid] = p;
          S.vj[par ^ 1][tid] = val;
          par ^= 1;
        }
        if (li < m) S.V[li] = val;  // x, in place
        bar_d();
      }
    }
    if (tid == 0) trace_stamp(a, t, 6);
    fence_proxy_async_smem();  // S.V (generic-proxy writes) → the bulk store
    if (bar_d_or(bad)) {
      if (tid == 0) record_error(ctx, DERR_CORRUPT);
    } else if (m % 2 == 0) {
      if (tid == 0) {
        tma_store_1d(out + t0, S.V, 8 * m);
        tma_store_commit();
      }
    } else {  // ragged last tile: thread stores
      for (uint32_t i = tid; i < m; i += kDT) __stcs(out + t0 + i, S.V[i]);
      __threadfence();
      bar_d();
    }
    pending = t;  // tile complete (also when malformed) once thread 0 has waited
  }
}

__global__ void __launch_bounds__(kDDecThreads) dpratio_decode_kernel(DecArgs a, LaunchCtx ctx) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  DDecSmem& S = *reinterpret_cast<DDecSmem*>(smem_raw);
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    mbar_init(&S.full_in[0], 1);
    mbar_init(&S.empty_in[0], kDW);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == 0) d_dec_loader(S, a, ctx, lane);
  else d_dec_compute(S, a, ctx, threadIdx.x - 32);
}

}  // namespace

// ---- host side -------------------------------------------------------------------
size_t dpratio_fcm_workspace(uint64_t n) { return fcm_dist_workspace(n); }

int launch_dpratio_encode(const EncArgs& a0, const LaunchCtx& ctx, void* ws, size_t ws_bytes, cudaStream_t st) {
  const uint64_t n = a0.n_words_total;
  int launches = 0;
  if (n) {
    uint32_t* dist = nullptr;  // FCM distances (L170–185), lcf_fcm.cu
    launches += launch_fcm_dist(reinterpret_cast<const uint64_t*>(a0.in), n, ws, ws_bytes, st, &dist);
    EncArgs a = a0;
    a.fcm_dist = dist;
    const size_t smem = sizeof(DEncSmem);
    static const bool init = [&] {
      cudaFuncSetAttribute(dpratio_encode_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      return true;
    }();
    (void)init;
    const int grid = persistent_grid(dpratio_encode_kernel, kDEncThreads, smem, a.n_chunks / 2);
    KTrace kt("dpratio_encode", st);
    dpratio_encode_kernel<<<grid, kDEncThreads, smem, st>>>(a, ctx);
    ++launches;
  }
  return launches;
}

void launch_dpratio_decode(const DecArgs& a, const LaunchCtx& ctx, uint64_t max_tiles, cudaStream_t st) {
  const size_t smem = sizeof(DDecSmem);
  static const bool init = [&] {
    cudaFuncSetAttribute(dpratio_decode_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    return true;
  }();
  (void)init;
  const int grid = persistent_grid(dpratio_decode_kernel, kDDecThreads, smem, (max_tiles + kDBatch - 1) / kDBatch);
  KTrace kt("dpratio_decode", st);
  dpratio_decode_kernel<<<grid, kDDecThreads, smem, st>>>(a, ctx);
}

}  // namespace lcf
