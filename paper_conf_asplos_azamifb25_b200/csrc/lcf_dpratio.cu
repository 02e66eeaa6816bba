// lcf_dpratio.cu — DPratio = per chunk (RARE ∘ RAZE ∘ DIFFMS₆₄) over FCM(x)
// (§3.2) on sm_100a.
//
// Compress: the FCM distances come from lcf_fcm.cu (the repo's own two-pass
// LSD radix sort of h | fp | i records, fcm_match's nearest same-hash
// candidates, fcm_verify in index order — L172–176, A-13..A-15); then
//   dpratio_encode   persistent pipeline (loader warp, storer warp, 8 compute
//                    warps); item = 2048-word tile t → chunk 2t (V) and 2t+1
//                    (Dist) (A-16); DIFFMS₆₄ in registers, RAZE → RARE planned
//                    from clz histograms (L201: shared atomics; k* from the
//                    prefix sums) and emitted by per-thread bit writers
// Decompress:
//   dpratio_decode   per tile: RARE⁻¹ → RAZE⁻¹ → DIFFMS⁻¹ for Dist and V, then
//                    the FCM decode of the tile (L197): references inside the
//                    tile by pointer jumping in shared memory, references into
//                    a completed earlier tile read its output; everything else
//                    is left PENDING (global target index + a bitmap bit) —
//                    no tile ever waits for another
//   dp_walk_nodes / dp_gather_leaves / dp_gather_nodes (one stream) or
//   dp_find_roots / dp_gather_roots (shards, peer streams through CUDA IPC):
//                    the pending words' roots by pointer walks with path
//                    compression (the paper's union-find "find"), then the
//                    values

#include "lcf_persist.cuh"

namespace lcf {
namespace {

constexpr int kDW = 8;                 // compute warps
constexpr uint32_t kDT = kDW * 32;     // compute threads
#ifndef LCF_DP_OUT
#define LCF_DP_OUT 2
#endif
constexpr int kDOut = LCF_DP_OUT, kDBatch = 4;  // output slots (encode), tiles per ticket (decode)
static_assert(kDOut >= 2, "a tile emits its V and Dist chunks into two slots (1 deadlocks; 3 measured equal)");
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
  return warp_uniform(r) != 0;  // (CTA-uniform; broadcast so that ptxas knows it)
}

// ============================ RAZE / RARE in shared memory ============================

__device__ __forceinline__ uint32_t clz64(uint64_t v) { return __clzll(v); }

// 64-bit field at bit position P of the little-endian word stream at `base`
// (4-byte aligned; reads up to 12 bytes; P < 2^32: shared-memory streams),
// masked by the caller's precomputed 2^w − 1 (all ones for w = 64, 0 for w = 0).
__device__ __forceinline__ uint64_t get_field_m(const uint32_t* base, uint32_t P, uint64_t mask) {
  const uint32_t* p = base + (P >> 5);
  const uint32_t r = P & 31;
  const uint32_t lo = __funnelshift_r(p[0], p[1], r), hi = __funnelshift_r(p[1], p[2], r);
  return (((uint64_t)hi << 32) | lo) & mask;
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
// shared-memory buffer. The run's first and last words may be shared with the
// neighbouring runs (OR-ed into a zeroed buffer); the words in between belong
// to this thread alone (plain stores). The pending partial word is 32 bits
// wide: a field of up to 64 bits completes at most two words, formed by funnel
// shifts. LCF_BW_PRED: put() is branch-free — both possible word writes are
// predicated shared stores / reductions, so lanes at different bit offsets do
// not diverge, and a field of width 0 is a no-op (callers pass w = 0 instead
// of skipping the call).
#ifndef LCF_BW_PRED
#define LCF_BW_PRED 1
#endif
__device__ __forceinline__ void sts_or_pred(uint32_t addr, uint32_t v, bool st, bool red) {
  asm volatile(
      "{\n .reg .pred ps, pr;\n setp.ne.u32 ps, %2, 0;\n setp.ne.u32 pr, %3, 0;\n"
      " @ps st.shared.u32 [%0], %1;\n @pr red.shared.or.b32 [%0], %1;\n}" ::"r"(addr),
      "r"(v), "r"((uint32_t)st), "r"((uint32_t)red)
      : "memory");
}
struct BitWriter {
  uint32_t* buf;
  uint32_t widx, w0, nb, pw;  // current word, first word, pending bits (< 32), pending word
  __device__ __forceinline__ BitWriter(uint32_t* b, uint64_t off)
      : buf(b), widx((uint32_t)(off >> 5)), w0((uint32_t)(off >> 5)), nb((uint32_t)(off & 31)), pw(0) {}
#if !LCF_BW_PRED
  __device__ __forceinline__ void out(uint32_t w) {
    if (widx == w0) atomicOr(buf + widx, w);
    else buf[widx] = w;
    ++widx;
  }
#endif
  // append the low w bits of f (f < 2^w, 0 ≤ w ≤ 64; w = 0 needs f = 0)
  __device__ __forceinline__ void put(uint64_t f, uint32_t w) {
    const uint32_t flo = (uint32_t)f, fhi = (uint32_t)(f >> 32);
    const uint32_t o0 = pw | (flo << nb);              // bits 0..31 of pw | f << nb
    const uint32_t o1 = __funnelshift_l(flo, fhi, nb);  // bits 32..63
    const uint32_t o2 = __funnelshift_l(fhi, 0u, nb);   // bits 64..95
    const uint32_t e = nb + w;
#if LCF_BW_PRED
    const bool c0 = e >= 32, c1 = e >= 64, first = widx == w0;
    const uint32_t a = smem_addr(buf + widx);
    sts_or_pred(a, o0, c0 && !first, c0 && first);
    sts_or_pred(a + 4, o1, c1, false);
    widx += (uint32_t)c0 + (uint32_t)c1;
    pw = c1 ? o2 : (c0 ? o1 : o0);
#else
    if (e >= 32) {
      out(o0);
      if (e >= 64) {
        out(o1);
        pw = o2;
      } else {
        pw = o1;
      }
    } else {
      pw = o0;
    }
#endif
    nb = e & 31;
  }
  __device__ __forceinline__ void finish() {
    if (nb) atomicOr(buf + widx, pw);
  }
};

// ---------------------------- RAZE / RARE encoder ----------------------------
// Thread t owns words 8t … 8t+7 of the stage's input (n ≤ 2048 words), held in
// registers: its B1 bits are B1 byte t, and its HI and LO fields are contiguous
// bit runs. A plan takes two CTA barriers; everything after the second one
// (the k choice, B2, B3, the section sizes) is computed redundantly by every
// warp from shared data, so no warp waits on another's serial work.
#ifndef LCF_ENC_MINB
#define LCF_ENC_MINB 3  // 64 registers, 48 B of spills: 3 CTAs/SM (density compress 1325 -> 1297 us, rt_density 1971 -> 1912 us)
#endif
struct EncScratch {
  uint32_t hist[2][66];  // clz histograms, alternating per plan; [65]: the tile has an FCM distance
  uint32_t b1[64];       // B1 bitmap; byte t = thread t's words
  uint32_t wtot[kDW];    // set words per warp
};

// 0x00/0xFF bytes → 4 bits (byte j → bit j)
__device__ __forceinline__ uint32_t bits4(uint32_t m) { return ((m & 0x01010101u) * 0x01020408u) >> 24; }

struct APlan {
  uint32_t n, tl, k, byte, rank0, c1m, off1, nr1, b3, hib, total;
  bool bypass, allzero, anyd;
};

// Plan of RAZE (RARE = false, L189) or RARE (RARE = true, L195) over the L-byte
// input whose words 8·tid … 8·tid+7 are v (0 at or past n = L/8) and whose
// word 8·tid − 1 is p (RARE's reference of v[0]; 0 for tid 0). Before its first
// barrier it also zeroes the other histogram and `zn` 16-byte words at zp.
// `dflag`: this thread saw an FCM distance (reported as anyd). A-17, A-18.
template <bool RARE>
__device__ __forceinline__ APlan a_plan(const uint64_t (&v)[8], uint64_t p, uint32_t L, EncScratch& sc,
                                        uint32_t par, uint32_t tid, bool dflag, uint4* zp, uint32_t zn) {
  const uint32_t warp = tid >> 5, lane = tid & 31;
  APlan P;
  P.n = L / 8;
  P.tl = L % 8;
  const uint32_t n = P.n, i0 = 8 * tid;
  uint32_t* H = sc.hist[par];
  // z_j = clz(v_j ⊕ ref_j) as bytes (0xFF past n): B1 bit j is [z_j < k] for
  // RAZE (top(v) ≠ 0) and RARE (top(v_j) ≠ top(v_{j−1})) alike
  uint32_t zpk[2] = {0u, 0u};
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    const uint64_t ref = RARE ? (j ? v[j - 1] : p) : 0ull;
    const uint32_t z = i0 + j < n ? clz64(v[j] ^ ref) : 0xFFu;
    if (z <= 64) atomicAdd(&H[z], 1u);
    zpk[j >> 2] |= z << (8 * (j & 3));
  }
  if (__any_sync(0xFFFFFFFFu, dflag) && lane == 0) atomicOr(&H[65], 1u);
  if (tid < 66) sc.hist[par ^ 1][tid] = 0;  // read by the previous plan before a later barrier
  for (uint32_t j = tid; j < zn; j += kDT) zp[j] = make_uint4(0, 0, 0, 0);
  bar_d();
  // ---- k* = smallest argmin of est(k) = k·nz(k) + (64−k)·n, k ∈ 1..64 (every warp) ----
  const uint32_t c0 = H[2 * lane], c1 = H[2 * lane + 1];
  P.allzero = H[64] == n;
  P.anyd = H[65] != 0;
  uint32_t s = c0 + c1;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, s, d);
    if ((int)lane >= d) s += y;
  }
  {
    const uint32_t before = s - c0 - c1;
    const uint32_t kA = 2 * lane + 1, kB = 2 * lane + 2;  // nz(kA) = before + c0, nz(kB) = s
    const uint32_t eA = kA * (before + c0) + (64 - kA) * n, eB = kB * s + (64 - kB) * n;
    const uint32_t keyA = (eA << 7) | kA, keyB = (eB << 7) | kB;
    const uint32_t best = __reduce_min_sync(0xFFFFFFFFu, keyA < keyB ? keyA : keyB);
    P.k = best & 127;
    // the fields alone (est(k*) bits) already reach the bypass size: bypass,
    // whatever the bitmaps add (A-23)
    P.bypass = 3 + ((best >> 7) + 7) / 8 + P.tl + ((((n + 7) / 8 + 7) / 8 + 7) / 8) >= 3 + L;
  }
  if (!RARE && P.allzero) return P;  // the caller writes the fixed stream
  if (P.bypass) return P;
  const uint32_t k = P.k, sh = 64 - k;  // top(v) = v >> sh (k = 64: sh = 0)
  // ---- B1 byte t = this thread's set bits; ranks of the set words ----
  (void)sh;
  const uint32_t kk = k * 0x01010101u;
  const uint32_t byte = bits4(__vcmpltu4(zpk[0], kk)) | (bits4(__vcmpltu4(zpk[1], kk)) << 4);
  P.byte = byte;
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
  uint32_t base = 0, nset = 0;
#pragma unroll
  for (uint32_t w = 0; w < kDW; ++w) {
    const uint32_t t = sc.wtot[w];
    base += w < warp ? t : 0u;
    nset += t;
  }
  P.rank0 = base + x - c;
  // ---- B1 → B2 → B3 (lane l: B1 bytes [8l, 8l+8) = words 2l, 2l+1 → B2 byte l) ----
  const uint32_t L1 = (n + 7) / 8, L2 = (L1 + 7) / 8, L3 = (L2 + 7) / 8;
  const uint32_t b1w0 = sc.b1[2 * lane], b1w1 = sc.b1[2 * lane + 1];
  const uint32_t prevb = __shfl_up_sync(0xFFFFFFFFu, b1w1 >> 24, 1);
  const uint32_t pre0 = (b1w0 << 8) | (lane ? prevb : 0u), pre1 = (b1w1 << 8) | (b1w0 >> 24);
  const uint32_t vb = 8 * lane >= L1 ? 0u : (L1 - 8 * lane >= 8 ? 0xFFu : (1u << (L1 - 8 * lane)) - 1u);
  const uint32_t c1m = (bits4(__vcmpne4(b1w0, pre0)) | (bits4(__vcmpne4(b1w1, pre1)) << 4)) & vb;
  uint32_t y = __popc(c1m);
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(0xFFFFFFFFu, y, d);
    if ((int)lane >= d) y += o;
  }
  P.c1m = c1m;  // B2 byte `lane`
  P.off1 = y - __popc(c1m);
  P.nr1 = __shfl_sync(0xFFFFFFFFu, y, 31);
  const uint32_t pb2 = __shfl_up_sync(0xFFFFFFFFu, c1m, 1);
  P.b3 = __ballot_sync(0xFFFFFFFFu, lane < L2 && c1m != (lane ? pb2 : 0u));
  P.hib = (nset * k + 7) / 8;
  const uint32_t lob = (n * (64 - k) + 7) / 8;
  P.total = 3 + P.hib + lob + P.tl + P.nr1 + __popc(P.b3) + L3;
  P.bypass = P.total >= 3 + L;  // A-23
  return P;
}

// Writes the planned (non-bypass) stream into dst, which is zero over its
// first P.total bytes: fields by per-thread bit writers, the header, tail,
// nr(B1), nr(B2) and B3 bytes as byte ORs. `tail` = the input's last L mod 8
// bytes. No barrier: the caller orders dst's readers after it.
__device__ __forceinline__ void a_emit(const uint64_t (&v)[8], const APlan& P, uint32_t L, const uint8_t* tail,
                                       uint8_t* dst, const EncScratch& sc, uint32_t tid) {
  const uint32_t warp = tid >> 5, lane = tid & 31;
  const uint32_t n = P.n, tl = P.tl, k = P.k, sh = 64 - k, wl = 64 - k, i0 = 8 * tid;
  uint32_t* dw = reinterpret_cast<uint32_t*>(dst);
  // ---- HI: top fields of the set words (rank order), LO: low fields of all words ----
  if (P.byte) {
    BitWriter bw(dw, 24 + (uint64_t)P.rank0 * k);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const bool on = (P.byte >> j) & 1;
      if (LCF_BW_PRED) bw.put(on ? v[j] >> sh : 0ull, on ? k : 0u);
      else if (on) bw.put(v[j] >> sh, k);
    }
    bw.finish();
  }
  if (wl && i0 < n) {
    const uint64_t lmask = (1ull << wl) - 1;  // wl ≤ 63
    BitWriter bw(dw, 8ull * (3 + P.hib) + (uint64_t)i0 * wl);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const bool on = i0 + j < n;
      if (LCF_BW_PRED) bw.put(on ? v[j] & lmask : 0ull, on ? wl : 0u);
      else if (on) bw.put(v[j] & lmask, wl);
    }
    bw.finish();
  }
  auto put_byte = [&](uint32_t pos, uint32_t val) { atomicOr(dw + (pos >> 2), (val & 0xFFu) << (8 * (pos & 3))); };
  const uint32_t after = 3 + P.hib + (n * wl + 7) / 8;
  if (tid == 0) atomicOr(dw, (L & 0xFFFFu) | (k << 16));
  if (tid < tl) put_byte(after + tid, tail[tid]);
  if (warp == kDW - 1) {  // nr(B1), nr(B2), B3
    const uint32_t L3 = (((n + 7) / 8 + 7) / 8 + 7) / 8;
    const uint32_t b1w0 = sc.b1[2 * lane], b1w1 = sc.b1[2 * lane + 1];
    uint32_t q = after + tl + P.off1;
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if ((P.c1m >> j) & 1) put_byte(q++, (j < 4 ? b1w0 : b1w1) >> (8 * (j & 3)));
    if ((P.b3 >> lane) & 1) put_byte(after + tl + P.nr1 + __popc(P.b3 & ((1u << lane) - 1)), P.c1m);
    if (lane < L3) put_byte(P.total - L3 + lane, P.b3 >> (8 * lane));
  }
}

// RAZE bypass from registers (A-23): u16 L ‖ u8 0 ‖ the input words, into a
// zeroed dst.
__device__ __forceinline__ void a_emit_bypass_regs(const uint64_t (&v)[8], uint32_t n, uint8_t* dst, uint32_t tid) {
  uint32_t* dw = reinterpret_cast<uint32_t*>(dst);
  const uint32_t i0 = 8 * tid;
  if (tid == 0) atomicOr(dw, (8 * n) & 0xFFFFu);
  if (i0 < n) {
    BitWriter bw(dw, 24 + 64ull * i0);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const bool on = i0 + j < n;
      if (LCF_BW_PRED) bw.put(on ? v[j] : 0ull, on ? 64u : 0u);
      else if (on) bw.put(v[j], 64);
    }
    bw.finish();
  }
}

// RARE bypass from shared memory: dst[0..3) = u16 L ‖ u8 0, dst[3 + j] = src[j].
// Four output words per thread per step (one 16-byte store, funnel shifts over
// a 16-byte load and the word before it); words past the stream are 0.
__device__ __forceinline__ void a_emit_bypass_smem(const uint8_t* src, uint32_t L, uint8_t* dst, uint32_t tid) {
  const uint32_t* sw = reinterpret_cast<const uint32_t*>(src);
  const uint32_t nw = (L + 3 + 3) / 4;  // output words
  for (uint32_t g = tid; 4 * g < nw; g += kDT) {
    const uint32_t w = 4 * g;
    const uint4 q = reinterpret_cast<const uint4*>(src)[g];  // src words w .. w+3 (slack-safe)
    const uint32_t pw = w ? sw[w - 1] : 0u;
    uint32_t o[4] = {__funnelshift_r(pw, q.x, 8), __funnelshift_r(q.x, q.y, 8), __funnelshift_r(q.y, q.z, 8),
                     __funnelshift_r(q.z, q.w, 8)};
    if (w == 0) o[0] = (L & 0xFFFFu) | (q.x << 24);
    if (w + 4 >= nw) {  // the group holding the stream's last word: mask past it
#pragma unroll
      for (uint32_t i = 0; i < 4; ++i) {
        const uint32_t keep = w + i < nw ? 3 + L - 4 * (w + i) : 0;  // bytes of this word inside the output
        if (keep < 4) o[i] &= keep ? (1u << (8 * keep)) - 1u : 0u;
      }
    }
    reinterpret_cast<uint4*>(dst)[g] = make_uint4(o[0], o[1], o[2], o[3]);
  }
}

// CTA-wide exclusive scan of u64 over the kDT compute threads. The warp sums go
// to slot sh[sp] and sp flips, so consecutive scans need no trailing barrier.
__device__ __forceinline__ uint64_t cta_scan_u64(uint64_t v, uint64_t (*sh)[kDW], uint32_t& sp, uint32_t tid,
                                                 uint64_t& total) {
  const uint32_t warp = tid >> 5, lane = tid & 31;
  uint64_t x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint64_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
    if ((int)lane >= d) x += y;
  }
  uint64_t* s = sh[sp];
  sp ^= 1;
  if (lane == 31) s[warp] = x;
  bar_d();
  uint64_t base = 0;
  total = 0;
#pragma unroll
  for (uint32_t i = 0; i < kDW; ++i) {
    const uint64_t t = s[i];
    if (i < warp) base += t;
    total += t;
  }
  return base + x - v;
}

// Decode a RAZE/RARE stream of `len` bytes at src (16-byte aligned, ≥ 16 bytes
// of readable slack) into dst (8-byte aligned, capacity cap). Returns the
// decoded length or −1 if malformed. All kDT compute threads call it. Every
// warp rebuilds B1 from B3 → B2 → B1 itself (lane l: B1 words 2l, 2l+1 and
// their set-word prefixes), so the only barrier is the one after dst.
// FUSE (RAZE⁻¹ of a DIFFMS stream, raze_diffms_inv): the words go straight
// into DIFFMS⁻¹ (see there); −2 = a bypassed stream, left to the plain path.
template <bool FUSE = false>
__device__ int adaptive_decode(const uint8_t* base, uint32_t off, uint32_t len, uint8_t* dst, uint32_t cap, bool rare,
                               uint32_t tid, uint64_t (*scan)[kDW] = nullptr, uint32_t* sp = nullptr,
                               uint64_t* any = nullptr) {
  const uint32_t warp = tid >> 5, lane = tid & 31;
  const uint8_t* src = base + off;  // the stream (base: 4-byte aligned)
  if (len < 3) return -1;
  const uint32_t L = src[0] | ((uint32_t)src[1] << 8), k = src[2];
  if (L > cap) return -1;
  if (k == 0) {  // bypass: dst[j] = src[3 + j], one funnel shift per word
    if (FUSE) return -2;  // (the caller decodes it unfused)
    if (len != 3 + L) return -1;
    const uint32_t* sw = reinterpret_cast<const uint32_t*>(base) + (off + 3) / 4;
    const uint32_t fs = 8 * ((off + 3) % 4);
    uint32_t* dw = reinterpret_cast<uint32_t*>(dst);
    for (uint32_t w = tid; w < (L + 3) / 4; w += kDT) dw[w] = __funnelshift_r(sw[w], sw[w + 1], fs);
    bar_d();
    return (int)L;
  }
  if (k > 64) return -1;
  const uint32_t n = L / 8, tl = L % 8, L1 = (n + 7) / 8, L2 = (L1 + 7) / 8, L3 = (L2 + 7) / 8;
  const uint32_t wl = 64 - k;
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
  const uint32_t cw0 = __popc(w0), cw1 = __popc(w1);
  uint32_t c = cw0 + cw1;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, c, d);
    if ((int)lane >= d) c += y;
  }
  const uint32_t cnt0 = c - cw0 - cw1, cnt1 = c - cw1;  // set words before B1 words 2l, 2l+1
  const uint32_t nset = __shfl_sync(0xFFFFFFFFu, c, 31);
  const uint32_t hib = (nset * k + 7) / 8, lob = (n * wl + 7) / 8;
  if (!bad && (int32_t)(3 + hib + lob + tl) != s1) bad = 1;
  if (bad) return -1;  // (warp-uniform, and the same in every warp)
  const uint32_t* sw = reinterpret_cast<const uint32_t*>(base);
  const uint32_t f0 = 8 * off;  // bit position of the stream in base (< 2^20: shared memory)
  const uint32_t lo_base = f0 + 8 * (3 + hib);
  const uint64_t hmask = k >= 64 ? ~0ull : (1ull << k) - 1, lmask = wl ? (1ull << wl) - 1 : 0ull;
  if constexpr (FUSE) {
    // RAZE⁻¹ fused with DIFFMS⁻¹ (no tail, L = cap = 8m): thread t decodes
    // words 8t … 8t+7 — B1 byte t, from lane t/8's B1 words — straight into
    // registers, unTCMS, then the CTA scan; dst receives the final words
    // after the scan's barrier (no round trip through dst before it)
    if (L != cap || tl) return -1;  // (uniform)
    const uint32_t sl = tid >> 3;
    const uint32_t a0 = __shfl_sync(0xFFFFFFFFu, w0, sl), a1 = __shfl_sync(0xFFFFFFFFu, w1, sl);
    const uint32_t e0 = __shfl_sync(0xFFFFFFFFu, cnt0, sl), e1 = __shfl_sync(0xFFFFFFFFu, cnt1, sl);
    const bool odd = (tid >> 2) & 1;
    const uint32_t bw = odd ? a1 : a0, sh8 = 8 * (tid & 3);
    const uint32_t byte = (bw >> sh8) & 0xFFu;
    uint32_t re = (odd ? e1 : e0) + __popc(bw & ((1u << sh8) - 1u));  // set words before word 8t
    uint64_t v[8], run = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const uint32_t i = 8 * tid + j;
      const bool set = (byte >> j) & 1;
      const uint64_t tp = set ? get_field_m(sw, f0 + 24 + re * k, hmask) : 0;
      re += set;
      const uint64_t lw = get_field_m(sw, lo_base + i * wl, lmask);
      v[j] = i < n ? tcms_inv((tp << wl) | lw) : 0;
      run += v[j];
    }
    uint64_t tot;
    uint64_t acc = cta_scan_u64(run, scan, *sp, tid, tot);
    uint64_t an = 0;
    uint64_t* arr = reinterpret_cast<uint64_t*>(dst);
#pragma unroll
    for (int j = 0; j < 8; j += 2) {
      const uint64_t x0 = acc + v[j], x1 = x0 + v[j + 1];
      acc = x1;
      reinterpret_cast<ulonglong2*>(arr)[4 * tid + j / 2] = make_ulonglong2(x0, x1);  // words ≥ m: scratch
      if (8 * tid + j < n) an |= x0;
      if (8 * tid + j + 1 < n) an |= x1;
    }
    *any = an;
    return (int)L;
  }
  // word i = 32·(B1 word index) + lane: B1 word q = 8r + warp covers i = 256 r + 32 warp + lane;
  // q's parity is the warp's (kDW even), so the source register is warp-uniform
  static_assert(kDW % 2 == 0, "B1 word parity = warp parity");
  const uint32_t wsel = (warp & 1) ? w1 : w0, csel = (warp & 1) ? cnt1 : cnt0;
#pragma unroll
  for (int r8 = 0; r8 < 8; ++r8) {
    const uint32_t i = tid + kDT * r8;
    const uint32_t q = r8 * kDW + warp;
    const uint32_t bw = __shfl_sync(0xFFFFFFFFu, wsel, q >> 1);
    const uint32_t re = __shfl_sync(0xFFFFFFFFu, csel, q >> 1) + __popc(bw & ((1u << lane) - 1));  // set words before i
    const bool set = (bw >> lane) & 1;
    if (i < n) {
      uint64_t tp;
      if (rare) {
        const uint32_t ri = re + set;  // set words up to and including i
        tp = ri ? get_field_m(sw, f0 + 24 + (ri - 1) * k, hmask) : 0;
      } else {
        tp = set ? get_field_m(sw, f0 + 24 + re * k, hmask) : 0;
      }
      const uint64_t lw = get_field_m(sw, lo_base + i * wl, lmask);  // (0 for k = 64)
      *reinterpret_cast<uint64_t*>(dst + 8 * i) = (tp << wl) | lw;
    }
  }
  if (tid < tl) dst[8 * n + tid] = base[lo_base / 8 + (n * wl + 7) / 8 + tid];
  bar_d();
  return (int)L;
}

// =================================== encode ======================================
struct DEncSmem {
  alignas(128) uint64_t xin[kTileWords];        // stage: x tile
  alignas(128) uint32_t din[kTileWords];        // stage: FCM distances of the tile
  alignas(128) uint8_t rz[kChunkBytes + 128];   // RAZE output (zero past what the last RAZE wrote)
  alignas(128) uint32_t out[kDOut][(kChunkBytes + 128) / 4];  // output slots (handed back zeroed)
  uint64_t full_in[1], empty_in[1], full_out[kDOut], empty_out[kDOut];
  uint64_t in_chunk[1], out_chunk[kDOut];
  uint32_t out_len[kDOut], out_raw[kDOut];
  uint64_t scan[2][kDW];  // cta_scan_u64 slots (alternating)
  alignas(16) uint8_t zc[64];  // the Dist chunk of a full tile without distances: its stream, once made
  uint32_t zlen;               // (0 = not yet)
  EncScratch sc;
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
  const uint32_t i0 = 8 * tid;
  uint32_t oit = 0;       // output-slot iteration (two chunks per tile)
  uint32_t par = 0;       // histogram parity
  uint32_t rz_used = 0;   // bytes of S.rz written by the last RAZE (re-zeroed by the next plan)
  for (uint32_t it = 0;; ++it) {
    mbar_wait(&S.full_in[0], it & 1);
    const uint64_t t = S.in_chunk[0];
    if (t == kNoChunk) {
      enc_forward_end<kDOut, 1>(S, oit, warp, lane);
      return;
    }
    const uint32_t m = (uint32_t)umin64(kTileWords, a.n_words_total - t * kTileWords);
    // ---- FCM outputs (L170–185) and DIFFMS₆₄ (L187) of V in registers: words 8·tid … 8·tid+7 ----
    uint64_t w[8];
    uint32_t dprev = 0, dor = 0;
    {
      uint64_t x[8];
      uint32_t d[8];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const ulonglong2 xx = reinterpret_cast<const ulonglong2*>(S.xin)[4 * tid + q];
        x[2 * q] = xx.x;
        x[2 * q + 1] = xx.y;
      }
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const uint4 dd = reinterpret_cast<const uint4*>(S.din)[2 * tid + q];
        d[4 * q] = dd.x;
        d[4 * q + 1] = dd.y;
        d[4 * q + 2] = dd.z;
        d[4 * q + 3] = dd.w;
      }
      uint64_t prev = 0;
      if (tid && i0 - 1 < m) {
        dprev = S.din[i0 - 1];
        prev = dprev ? 0ull : S.xin[i0 - 1];
      }
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const bool in = i0 + j < m;
        if (!in) d[j] = 0;
        const uint64_t cur = d[j] ? 0ull : x[j];
        w[j] = in ? tcms((uint64_t)(cur - prev)) : 0ull;
        prev = cur;
        dor |= d[j];
      }
    }
    // the stage has been read: hand it back so the next tile loads during this one
    __syncwarp();
    if (lane == 0) mbar_arrive(&S.empty_in[0]);
    bool dist_zero = false;  // the tile has no FCM match (set by part 0's plan)
    for (uint32_t part = 0; part < 2; ++part, ++oit) {  // chunk 2t: V, chunk 2t+1: Dist (A-16)
      const uint64_t c = 2 * t + part;
      if (tid == 0) trace_stamp(a, c, 1);
      const uint32_t o = oit % kDOut, pho = (oit / kDOut) & 1;
      uint8_t* ob = reinterpret_cast<uint8_t*>(S.out[o]);
      const bool cacheable = part == 1 && dist_zero && m == kTileWords;
      if (cacheable && S.zlen) continue;  // written with the V chunk (below)
      const uint32_t* gd = a.fcm_dist + t * kTileWords;  // (the stage is gone: distances from L2)
      if (part == 1) {  // DIFFMS₆₄ of the distances
        uint64_t pd = dprev;
        uint32_t dv[8];
        if (i0 + 8 <= m) {  // two 16-byte loads per thread (the tile's distances are 16-byte aligned)
          const uint4 q0 = __ldcg(reinterpret_cast<const uint4*>(gd + i0));
          const uint4 q1 = __ldcg(reinterpret_cast<const uint4*>(gd + i0) + 1);
          dv[0] = q0.x; dv[1] = q0.y; dv[2] = q0.z; dv[3] = q0.w;
          dv[4] = q1.x; dv[5] = q1.y; dv[6] = q1.z; dv[7] = q1.w;
        } else {
#pragma unroll
          for (int j = 0; j < 8; ++j) dv[j] = i0 + j < m ? __ldcg(gd + i0 + j) : 0u;
        }
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const uint64_t dj = dv[j];
          w[j] = tcms(dj - pd);
          pd = dj;
        }
      }
      // ---- RAZE (L189) into S.rz ----
      const APlan P1 = a_plan<false>(w, 0ull, 8 * m, S.sc, par, tid, part == 0 && dor != 0,
                                     reinterpret_cast<uint4*>(S.rz), (rz_used + 8 + 15) / 16);
      par ^= 1;
      if (part == 0) dist_zero = !P1.anyd;
      uint32_t l1;
      if (P1.allzero) {
        // all-zero DIFFMS words (e.g. the Dist chunk of a tile without FCM
        // matches): k = 64, B1..B3 are zero and nothing repeats — the stream is
        // L | k=64 | L3 zero bytes (FORMAT.md §6.2, what a_emit would write)
        const uint32_t L = 8 * m, L3 = (((m + 7) / 8 + 7) / 8 + 7) / 8;
        if (tid < 3) S.rz[tid] = tid == 0 ? (uint8_t)L : tid == 1 ? (uint8_t)(L >> 8) : 64;
        l1 = 3 + L3;
      } else if (P1.bypass) {
        a_emit_bypass_regs(w, m, S.rz, tid);
        l1 = 3 + 8 * m;
      } else {
        a_emit(w, P1, 8 * m, nullptr, S.rz, S.sc, tid);
        l1 = P1.total;
      }
      rz_used = l1;
      bar_d();  // S.rz complete
      // ---- RARE (L195) of the RAZE stream; planned first, so the chunk's size —
      // and its aggregate for the look-back of later chunks — is known before an
      // output slot is needed ----
      uint64_t r[8];
      load8(reinterpret_cast<const uint64_t*>(S.rz), l1 / 8, tid, r);
      const uint64_t rp = (tid && i0 - 1 < l1 / 8) ? reinterpret_cast<const uint64_t*>(S.rz)[i0 - 1] : 0ull;
      const APlan P2 = a_plan<true>(r, rp, l1, S.sc, par, tid, false, nullptr, 0);
      par ^= 1;
      const uint32_t l2 = P2.bypass ? 3 + l1 : P2.total;
      const uint32_t raw_len = 8 * m;
      const bool raw = l2 >= raw_len;  // L104, ties → raw
      const uint32_t len = raw ? raw_len : l2;
      if (tid == 0) {
        lookback_publish(ctx, c, round16(len));
        trace_stamp(a, c, 2);
      }
      mbar_wait(&S.empty_out[o], pho ^ 1);  // (the storer hands slots back zeroed)
      if (tid == 0) trace_stamp(a, c, 3);
      if (raw) {  // the V / Dist words themselves, rebuilt from x and the distances (L2)
        uint64_t* ow = reinterpret_cast<uint64_t*>(ob);
        const uint64_t* gx = reinterpret_cast<const uint64_t*>(a.in) + t * kTileWords;
        for (uint32_t i = tid; i < m; i += kDT) {
          const uint32_t di = __ldcg(gd + i);
          ow[i] = part ? (uint64_t)di : (di ? 0ull : __ldcg(gx + i));
        }
        if (tid < 2 && (m & 1)) ow[m + tid] = 0;  // round16 pad
      } else if (P2.bypass) {
        a_emit_bypass_smem(S.rz, l1, ob, tid);
      } else {
        a_emit(r, P2, l1, S.rz + 8 * P2.n, ob, S.sc, tid);
      }
      if (cacheable && !raw && round16(len) <= sizeof(S.zc)) {  // remember it (read after later barriers)
        bar_d();
        if (tid < round16(len)) S.zc[tid] = ob[tid];
        if (tid == 0) S.zlen = len;
      }
      if (tid == 0) {
        S.out_chunk[o] = c;
        S.out_len[o] = len;
        S.out_raw[o] = raw;
      }
      // the next chunk — this tile's Dist — is the all-zero chunk whose stream
      // this CTA already holds: it goes into the next slot now, under the same
      // barrier (uniform: dist_zero and S.zlen are read after barriers)
      const bool zd = part == 0 && dist_zero && m == kTileWords && S.zlen != 0;
      const uint32_t o2 = (oit + 1) % kDOut, pho2 = ((oit + 1) / kDOut) & 1;
      if (zd) {
        const uint32_t zl = S.zlen;
        if (tid == 0) lookback_publish(ctx, c + 1, round16(zl));
        mbar_wait(&S.empty_out[o2], pho2 ^ 1);
        if (tid < round16(zl) / 4) S.out[o2][tid] = reinterpret_cast<const uint32_t*>(S.zc)[tid];
        if (tid == 0) {
          S.out_chunk[o2] = c + 1;
          S.out_len[o2] = zl;
          S.out_raw[o2] = 0;
        }
      }
      fence_proxy_async_smem();
      bar_d();
      if (tid == 0) trace_stamp(a, c, 4);
      if (lane == 0) {
        mbar_arrive(&S.full_out[o]);
        if (zd) mbar_arrive(&S.full_out[o2]);
      }
    }
  }
}

__global__ void __launch_bounds__(kDEncThreads, LCF_ENC_MINB) dpratio_encode_kernel(EncArgs a, LaunchCtx ctx) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  DEncSmem& S = *reinterpret_cast<DEncSmem*>(smem_raw);
  const uint32_t warp = warp_index_uniform(), lane = threadIdx.x & 31;
  // invariants: both histograms, S.rz and the output slots start zeroed
  for (uint32_t i = threadIdx.x; i < 2 * 66; i += blockDim.x) (&S.sc.hist[0][0])[i] = 0;
  for (uint32_t i = threadIdx.x; i < sizeof(S.rz) / 16; i += blockDim.x)
    reinterpret_cast<uint4*>(S.rz)[i] = make_uint4(0, 0, 0, 0);
  for (uint32_t i = threadIdx.x; i < sizeof(S.out) / 16; i += blockDim.x)
    reinterpret_cast<uint4*>(&S.out[0][0])[i] = make_uint4(0, 0, 0, 0);
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
  else if (warp == 1) enc_storer<kDOut, 1, DEncSmem, false, true>(S, a, ctx, lane, 0);
  else d_enc_compute(S, a, ctx, threadIdx.x - 64);
}

// =================================== decode ======================================
// Four 16.5 KB buffers (3 CTAs per SM): the V payload stage sv (released right
// after V's RARE⁻¹), the Dist payload stage sd (which then holds the Dist
// words: raw in place, or RAZE⁻¹'s output), rz (RARE⁻¹ output of V, then of
// Dist; the FCM decode's pointer-jumping scratch) and X (V, then the decoded
// tile in place, stored by TMA).
struct DDecSmem {
  alignas(128) uint8_t sv[kChunkBytes + 128];
  alignas(128) uint8_t sd[kChunkBytes + 128];
  alignas(128) uint8_t rz[kChunkBytes + 128];
  alignas(128) uint64_t X[kTileWords + 8];
  uint32_t pmask[kTileWords / 32];  // shard decode: pending words of the tile
  uint64_t full_v[1], empty_v[1], full_d[1], empty_d[1];
  uint64_t tile[1];
  uint32_t len[2], flags[1];
  uint64_t scan[2][kDW];  // cta_scan_u64 slots (alternating)
};
struct FcmScratch {  // pointer jumping (aliases S.rz)
  int32_t pj[2][kDT];  // target (−1 done)
  uint64_t vj[2][kDT];
  uint8_t fj[2][kDT];  // value is a pending global target
};
static_assert(sizeof(FcmScratch) <= kChunkBytes, "FCM scratch fits in rz");

__device__ __forceinline__ void d_dec_loader(DDecSmem& S, const DecArgs& a, const LaunchCtx& ctx, uint32_t lane) {
  uint64_t n_words = 0, n_chunks = 0, base = 0, payload = 0;
  const bool hdr_ok = read_header(a, ctx, n_words, n_chunks, base, payload);
  const bool small = hdr_ok && n_words * 8 > a.out_capacity;
  const uint64_t T = a.end_tile && a.end_tile < n_chunks / 2 ? a.end_tile : n_chunks / 2;
  uint32_t it = 0;
  for (;;) {
    uint64_t tb = 0;
    if (lane == 0) tb = atomicAdd(ctx.ticket, 1ull);
    tb = a.first_tile + __shfl_sync(0xFFFFFFFFu, tb, 0) * kDBatch;
    if (!hdr_ok || small || tb >= T) {
      mbar_wait(&S.empty_v[0], (it & 1) ^ 1);
      if (lane == 0) {
        if (tb == a.first_tile && !hdr_ok) record_error(ctx, DERR_CORRUPT);
        if (tb == a.first_tile && small) record_error(ctx, DERR_SMALL);
        S.tile[0] = kNoChunk;
        mbar_arrive(&S.full_v[0]);
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
    // prefixes relative to the launch's first chunk; a.base_off makes them absolute
    const uint64_t base_b = lookback_warp(ctx, 2 * tb, __shfl_sync(0xFFFFFFFFu, agg, 0), 2 * a.first_tile);
    const uint64_t rel = base_b + x;
    if (lane > 0 && lane < 2 * nb) st_relaxed_u64(ctx.status + c, make_status(kFlagInc, ctx.epoch, rel + agg));
    const uint64_t excl = rel + a.base_off;
    const uint64_t end = excl + round16(len);
    if (lane < 2 * nb && !bad && (end > payload || (c == n_chunks - 1 && end != payload))) bad = true;
    for (uint32_t j = 0; j < nb; ++j, ++it) {
      const uint32_t l0 = __shfl_sync(0xFFFFFFFFu, len, 2 * j), l1 = __shfl_sync(0xFFFFFFFFu, len, 2 * j + 1);
      const uint32_t r0 = __shfl_sync(0xFFFFFFFFu, raw, 2 * j), r1 = __shfl_sync(0xFFFFFFFFu, raw, 2 * j + 1);
      const bool b0 = __shfl_sync(0xFFFFFFFFu, bad, 2 * j), b1 = __shfl_sync(0xFFFFFFFFu, bad, 2 * j + 1);
      const uint64_t e0 = __shfl_sync(0xFFFFFFFFu, excl, 2 * j), e1 = __shfl_sync(0xFFFFFFFFu, excl, 2 * j + 1);
      const bool bb = b0 || b1;
      if (lane == 0) trace_stamp(a, tb + j, 0);
      mbar_wait(&S.empty_v[0], (it & 1) ^ 1);
      if (lane == 0) {
        trace_stamp(a, tb + j, 1);
        if (bb) record_error(ctx, DERR_CORRUPT);
        S.tile[0] = tb + j;
        S.len[0] = l0;
        S.len[1] = l1;
        S.flags[0] = r0 | (r1 << 1) | (bb ? 4u : 0u);
        if (!bb && l0) {
          mbar_arrive_expect_tx(&S.full_v[0], (uint32_t)round16(l0));
          tma_load_1d(S.sv, a.stream + base + e0, (uint32_t)round16(l0), &S.full_v[0]);
        } else {
          mbar_arrive(&S.full_v[0]);
        }
      }
      mbar_wait(&S.empty_d[0], (it & 1) ^ 1);
      if (lane == 0) {
        if (!bb && l1) {
          mbar_arrive_expect_tx(&S.full_d[0], (uint32_t)round16(l1));
          tma_load_1d(S.sd, a.stream + base + e1, (uint32_t)round16(l1), &S.full_d[0]);
        } else {
          mbar_arrive(&S.full_d[0]);
        }
      }
    }
  }
}

// RAZE stream of an all-zero chunk (the encoder's fixed stream): k = 64 and
// nothing but L3 zero B3 bytes. Returns 1 if rz is exactly that, 0 if it is
// not of that shape, −1 if it has that shape with a non-zero B3 byte (any set
// B3 bit would claim nr(B2) bytes that are not there: malformed).
__device__ __forceinline__ int fixed_zero_stream(const uint8_t* rz, int l1, uint32_t m) {
  const uint32_t L = rz[0] | ((uint32_t)rz[1] << 8), n = L / 8;
  const uint32_t L3 = (((n + 7) / 8 + 7) / 8 + 7) / 8;
  if (!(l1 >= 3 && rz[2] == 64 && L == 8 * m && (uint32_t)l1 == 3 + L3)) return 0;
  for (uint32_t j = 0; j < L3; ++j)
    if (rz[3 + j]) return -1;
  return 1;
}

// RAZE⁻¹ of the stream at rz + off (length l1) into arr (m words) and
// DIFFMS⁻¹ in place (L94: the inverse stages in reverse order). Ends without a
// barrier after the scan; returns false if malformed.
__device__ __forceinline__ bool raze_diffms_inv(const uint8_t* rz, uint32_t off, int l1, uint32_t m, uint64_t* arr,
                                                uint64_t& any, DDecSmem& S, uint32_t& sp, uint32_t tid) {
#ifndef LCF_DEC_FUSE
#define LCF_DEC_FUSE 1
#endif
  if (LCF_DEC_FUSE) {
    const int lf = adaptive_decode<true>(rz, off, (uint32_t)l1, reinterpret_cast<uint8_t*>(arr), 8 * m, false, tid,
                                         S.scan, &sp, &any);
    if (lf != -2) return lf == (int)(8 * m);  // else a bypassed RAZE stream: below
  }
  const int l0 = adaptive_decode(rz, off, (uint32_t)l1, reinterpret_cast<uint8_t*>(arr), 8 * m, false, tid);
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
  uint64_t acc = cta_scan_u64(run, S.scan, sp, tid, tot);
  any = 0;
#pragma unroll
  for (int j = 0; j < 8; j += 2) {
    const uint64_t a0 = acc + v[j], a1 = a0 + v[j + 1];
    acc = a1;
    reinterpret_cast<ulonglong2*>(arr)[4 * tid + j / 2] = make_ulonglong2(a0, a1);  // words ≥ m: scratch
    if (8 * tid + j < m) any |= a0;
    if (8 * tid + j + 1 < m) any |= a1;
  }
  return true;
}

__device__ __forceinline__ void d_dec_compute(DDecSmem& S, const DecArgs& a, const LaunchCtx& ctx, uint32_t tid) {
  const uint32_t lane = tid & 31;
  const uint4 h0 = reinterpret_cast<const uint4*>(a.stream)[0];
  const uint64_t n_words = (((uint64_t)h0.w << 32) | h0.z) / 8;
  uint64_t* out = reinterpret_cast<uint64_t*>(a.out);
  // The decoded tile leaves S.X by a TMA bulk store issued by thread 0; its
  // completion (and the tile's flag) is awaited only before S.X is written
  // again, or at exit.
  uint64_t pending = kNoChunk;
  uint32_t sp = 0;  // cta_scan_u64 slot parity
  auto finish_pending = [&]() {
    if (tid == 0 && pending != kNoChunk) {
      tma_store_wait_all0();
      __threadfence();
      st_release_u32(a.tile_flag + pending, ctx.epoch);
      trace_stamp(a, pending, 7);
    }
    pending = kNoChunk;
  };
  auto release = [&](uint64_t* bar) {
    __syncwarp();
    if (lane == 0) mbar_arrive(bar);
  };
  FcmScratch& F = *reinterpret_cast<FcmScratch*>(S.rz);
  for (uint32_t it = 0;; ++it) {
    mbar_wait(&S.full_v[0], it & 1);
    const uint64_t t = warp_uniform(S.tile[0]);
    if (t == kNoChunk) {
      finish_pending();
      return;
    }
    const uint32_t fl = warp_uniform(S.flags[0]), lenV = warp_uniform(S.len[0]), lenD = warp_uniform(S.len[1]);
    const uint32_t m = (uint32_t)umin64(kTileWords, n_words - t * kTileWords);
    if (tid == 0) trace_stamp(a, t, 2);
    bool ok = !(fl & 4);
    const uint64_t t0 = t * kTileWords;
    // ---- Dist first: RARE⁻¹ → rz, RAZE⁻¹ → sd (a raw Dist chunk stays in sd) ----
    mbar_wait(&S.full_d[0], it & 1);
    const uint64_t* Dw = reinterpret_cast<const uint64_t*>(S.sd);
    bool nzD = false;
    if (ok && (fl & 2)) {
      uint64_t acc = 0;
      for (uint32_t i = tid; i < m; i += kDT) acc |= Dw[i];
      nzD = bar_d_or(acc != 0);
    } else if (ok) {
      const int l1D = adaptive_decode(S.sd, 0, lenD, S.rz, kChunkBytes + 3, true, tid);
      const int fz = l1D < 0 ? -1 : fixed_zero_stream(S.rz, l1D, m);
      if (fz < 0) {
        ok = false;
      } else if (!fz) {
        uint64_t any;
        ok = raze_diffms_inv(S.rz, 0, l1D, m, reinterpret_cast<uint64_t*>(S.sd), any, S, sp, tid);
        if (ok) nzD = bar_d_or(any != 0);
      }
    }
    // thread 0 waits for a previous bulk store out of X (only tiles with
    // distances use one); the barrier orders that and every read of rz before
    // V writes X and rz
    finish_pending();
    ok = !bar_d_or(!ok);
    if (!nzD) release(&S.empty_d[0]);
    if (tid == 0) trace_stamp(a, t, 3);
    // ---- V: RAZE⁻¹ → X and DIFFMS⁻¹ in X (the decoded tile leaves X by a TMA
    // bulk store) ----
    if (ok && (fl & 1)) {  // raw V chunk: the V words themselves
      const uint64_t* sw = reinterpret_cast<const uint64_t*>(S.sv);
      for (uint32_t i = tid; i < m; i += kDT) S.X[i] = sw[i];
      bar_d();
      release(&S.empty_v[0]);
    } else if (ok) {
      // RARE bypassed (k = 0, A-23): RAZE⁻¹ reads the stream in place at sv + 3;
      // otherwise RARE⁻¹ → rz first and sv is released right away
      const uint32_t L = S.sv[0] | ((uint32_t)S.sv[1] << 8);
      const bool inplace = lenV >= 3 && S.sv[2] == 0 && lenV == 3 + L;
      int l1V = (int)L;
      if (!inplace) {
        l1V = adaptive_decode(S.sv, 0, lenV, S.rz, kChunkBytes + 3, true, tid);
        ok = l1V >= 0;
        release(&S.empty_v[0]);
      }
      const uint8_t* zb = inplace ? S.sv : S.rz;
      const uint32_t zoff = inplace ? 3 : 0;
      if (ok) {
        const int fz = fixed_zero_stream(zb + zoff, l1V, m);
        if (fz < 0) {
          ok = false;
        } else if (fz) {  // DIFFMS⁻¹ of zeros
          for (uint32_t i = tid; i < m; i += kDT) S.X[i] = 0;
        } else {
          uint64_t any;
          ok = raze_diffms_inv(zb, zoff, l1V, m, S.X, any, S, sp, tid);
        }
      }
      if (inplace) {
        bar_d();  // every thread is past its reads of sv
        release(&S.empty_v[0]);
      }
    } else {
      release(&S.empty_v[0]);
    }
    if (tid == 0) trace_stamp(a, t, 4);
    if (tid == 0) trace_stamp(a, t, 5);
    // ---- FCM decode of the tile (L197): x[i] = Dist[i] ? x[i − Dist[i]] : V[i] ----
    // Chains inside the tile are followed here (pointer jumping in shared
    // memory). A reference into an earlier tile is read if that tile is
    // complete; otherwise — and for a word before the stream's first word
    // (shard decode) — the word is left PENDING: it holds the global index it
    // copies and its bit is set in a.pend. No tile ever waits for another:
    // dp_find_roots / dp_gather_roots (below) resolve the pending words after
    // this kernel, so long cross-tile chains (a value repeated row after row)
    // cost pointer jumps instead of a tile-by-tile serial dependency.
    bool bad = !ok;
    const uint64_t gb = a.gbase;  // global index of this stream's word 0
    if (ok && nzD) {  // (no distances: x = V as it stands)
      for (uint32_t w = tid; w < kTileWords / 32; w += kDT) S.pmask[w] = 0;
      bar_d();  // X complete (V's DIFFMS⁻¹ ends without a barrier)
      for (uint32_t b = 0; b < m; b += kDT) {  // 256-element blocks in index order
        const uint32_t li = b + tid;
        int32_t p = -1;
        uint64_t val = 0;
        uint8_t f = 0;  // val is a pending global target
        if (li < m) {
          const uint64_t d = Dw[li], gi = gb + t0 + li;
          if (d == 0) {
            val = S.X[li];
          } else if (d > gi || S.X[li] != 0) {
            bad = true;
          } else if (gi - d >= gb + t0 + b) {
            p = (int32_t)(gi - d - gb - t0 - b);  // inside this block: resolve below
          } else if (gi - d >= gb + t0) {
            const uint32_t lj = (uint32_t)(gi - d - gb - t0);
            val = S.X[lj];  // earlier block of this tile: final or pending
            f = (S.pmask[lj / 32] >> (lj % 32)) & 1;
          } else if (gi - d >= gb) {  // earlier tile of this stream
            const uint64_t j = gi - d - gb, tj = j / kTileWords;
            if (tj < a.first_tile) {  // an earlier launch on this stream: final
              val = ld_cg_u64(out + j);
            } else if (ld_acquire_u32(a.tile_flag + tj) == ctx.epoch) {  // complete: final or pending
              val = ld_cg_u64(out + j);
              f = (__ldcg(a.pend + j / 32) >> (j % 32)) & 1;
            } else {  // still in flight: pending on it
              val = gi - d;
              f = 1;
            }
          } else {  // before the shard: pending on the global word gi − d
            val = gi - d;
            f = 1;
          }
        }
        // pointer jumping inside the block (≤ 8 rounds; chains point backwards)
        uint32_t par = 0;
        F.pj[0][tid] = p;
        F.vj[0][tid] = val;
        F.fj[0][tid] = f;
        while (bar_d_or(p >= 0)) {
          if (p >= 0) {
            const int32_t q = F.pj[par][p];
            if (q < 0) {
              val = F.vj[par][p];
              f = F.fj[par][p];
              p = -1;
            } else {
              p = q;
            }
          }
          F.pj[par ^ 1][tid] = p;
          F.vj[par ^ 1][tid] = val;
          F.fj[par ^ 1][tid] = f;
          par ^= 1;
        }
        if (li < m) S.X[li] = val;  // x (or a pending target), in place
        {  // the warp's 32 consecutive words are one bitmap word (blocks start at multiples of 256)
          const uint32_t pm = __ballot_sync(0xFFFFFFFFu, li < m && f);
          if (lane == 0 && b + (tid & ~31u) < m) S.pmask[(b + (tid & ~31u)) / 32] = pm;
        }
        // mark the word a pending word points at (a chain node, walked first by
        // dp_find_roots); lanes hitting the same bitmap word send one OR
        const bool mk = li < m && f && val >= gb && val - gb < n_words;
        const uint32_t mkmask = __ballot_sync(0xFFFFFFFFu, mk);
        if (mk) {
          const uint64_t lt = val - gb;
          const uint32_t key = (uint32_t)(lt / 32), lead = __ffs(mkmask) - 1;
          const uint32_t key0 = __shfl_sync(mkmask, key, lead);
          if (__all_sync(mkmask, key == key0)) {  // the usual case: one bitmap word for the warp
            const uint32_t bitsum = __reduce_or_sync(mkmask, 1u << (lt % 32));
            if ((threadIdx.x & 31) == lead) {
              const uint32_t fresh = bitsum & ~atomicOr(a.tgt + key, bitsum);
              if (a.nodes && fresh) {  // first marks: onto the chain-node list
                uint32_t k = atomicAdd(a.n_nodes, (uint32_t)__popc(fresh));
                for (uint32_t b = fresh; b; b &= b - 1) a.nodes[k++] = 32 * key + (__ffs(b) - 1);
              }
            }
          } else {
            const uint32_t bit = 1u << (lt % 32);
            if (!(atomicOr(a.tgt + key, bit) & bit) && a.nodes) a.nodes[atomicAdd(a.n_nodes, 1u)] = (uint32_t)lt;
          }
        }
        bar_d();
      }
      // the tile's pending bits, before its completion flag (released after a barrier)
      for (uint32_t w = tid; w < (m + 31) / 32; w += kDT) {
        const uint32_t pm = bad ? 0u : S.pmask[w];
        a.pend[t0 / 32 + w] = pm;
        if (pm) st_relaxed_u32(a.any_pend, ctx.epoch);  // some word of this launch is pending
      }
      release(&S.empty_d[0]);
    } else {
      for (uint32_t w = tid; w < (m + 31) / 32; w += kDT) a.pend[t0 / 32 + w] = 0;
    }
    if (tid == 0) trace_stamp(a, t, 6);
    fence_proxy_async_smem();  // S.X (generic-proxy writes) → the bulk store
    if (bar_d_or(bad)) {
      if (tid == 0) record_error(ctx, DERR_CORRUPT);
    } else if (m % 2 == 0) {
      if (tid == 0) {
        tma_store_1d(out + t0, S.X, 8 * m);
        tma_store_commit();
      }
    } else {  // ragged last tile: thread stores
      for (uint32_t i = tid; i < m; i += kDT) __stcs(out + t0 + i, S.X[i]);
      __threadfence();
      bar_d();
    }
    pending = t;  // tile complete (also when malformed) once thread 0 has waited
  }
}

__global__ void __launch_bounds__(kDDecThreads, 3) dpratio_decode_kernel(DecArgs a, LaunchCtx ctx) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  DDecSmem& S = *reinterpret_cast<DDecSmem*>(smem_raw);
  const uint32_t warp = warp_index_uniform(), lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    mbar_init(&S.full_v[0], 1);
    mbar_init(&S.empty_v[0], kDW);
    mbar_init(&S.full_d[0], 1);
    mbar_init(&S.empty_d[0], kDW);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == 0) d_dec_loader(S, a, ctx, lane);
  else d_dec_compute(S, a, ctx, threadIdx.x - 32);
}

}  // namespace

// ---- host side -------------------------------------------------------------------
size_t dpratio_fcm_workspace(uint64_t n) { return fcm_dist_workspace(n); }

int launch_dpratio_encode(const EncArgs& a0, const LaunchCtx& ctx, void* ws, size_t ws_bytes, cudaStream_t st,
                          uint32_t halo, uint64_t gbase, const void* carry, bool sorted) {
  const uint64_t n = a0.n_words_total;
  int launches = 0;
  if (n) {
    uint32_t* dist = nullptr;  // FCM distances (L170–185), lcf_fcm.cu; a shard's with its carry
    const uint64_t* srt = nullptr;
    launches += launch_fcm_shard(reinterpret_cast<const uint64_t*>(a0.in), n, halo, gbase, carry, nullptr, true, ws,
                                 ws_bytes, st, &dist, sorted, &srt);
    EncArgs a = a0;
    a.fcm_dist = dist;
    (void)srt;
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

namespace {
// ---- root resolution of pending words (L197's union-find "find") ----------------
// After the tile decoder, a pending word holds the global index of the word it
// copies (always a smaller index). dp_find_roots follows each pending word's
// chain to its root — the first word on it that is not pending — and stores
// the root index in the word, writing the partial result back every few hops
// so that walks through it jump further (path compression, as the paper's
// decoder shortens chains for other threads). Every stored index is an
// ancestor on the chain, so a concurrent walker reading an old or a new value
// stays correct; no value is written until dp_gather_roots, after every walk
// has ended. Grid-stride in index order: earlier words are compressed first.
__device__ __forceinline__ int dp_owner(const DpViews& V, uint64_t g) {
  int q = (int)V.self;
  while (q > 0 && g < V.v[q].first) --q;
  return q;
}

__device__ __forceinline__ uint64_t dp_hi(const DpViews& V, const uint8_t* stream, uint64_t w_hi) {
  const DpView& me = V.v[V.self];
  uint64_t hi = w_hi < me.n ? w_hi : me.n;
  if (stream) {  // the stream's word count (a malformed header was reported by the decoder)
    const uint64_t nw = reinterpret_cast<const uint64_t*>(stream)[1] / 8;
    hi = hi < nw ? hi : nw;
  }
  return hi;
}

template <bool kSingle>
__global__ void __launch_bounds__(256) dp_find_roots_kernel(const __grid_constant__ DpViews V, const uint8_t* stream,
                                                           uint64_t w_lo, uint64_t w_hi, LaunchCtx ctx,
                                                           const uint32_t* any_pend, int mode) {
  if (any_pend && *any_pend != ctx.epoch) return;
  const DpView& me = V.v[V.self];
  const uint64_t hi = dp_hi(V, stream, w_hi);
  const uint32_t lane = threadIdx.x & 31;
  for (uint64_t base = w_lo + (blockIdx.x * 256ull + threadIdx.x - lane); base < hi; base += gridDim.x * 256ull) {
    uint32_t bits = __ldcg(me.pend + base / 32);  // one bitmap word per warp (w_lo % 32 == 0)
    if (!bits) continue;
    if (mode != 2) {
      const uint32_t nodes = __ldcg(me.tgt + base / 32);
      bits &= mode == 0 ? nodes : ~nodes;
    }
    const uint64_t li = base + lane;
    if (!((bits >> lane) & 1) || li >= hi) continue;
    uint64_t cur = me.first + li, t = __ldcg(me.out + li);
    bool err = false;
    for (;;) {
      if (t >= cur) { err = true; break; }  // chains point strictly backwards
      const DpView& w = V.v[kSingle ? 0 : dp_owner(V, t)];
      if (t < w.first || t - w.first >= w.n) { err = true; break; }
      const uint64_t lj = t - w.first;
      // the bit and the word are fetched together (one round trip per hop)
      uint32_t pw;
      uint64_t nt;
      if (kSingle) {
        pw = __ldcg(w.pend + lj / 32);
        nt = ld_relaxed_u64(w.out + lj);
      } else {
        pw = ld_relaxed_sys_u32(w.pend + lj / 32);
        nt = ld_relaxed_sys_u64(w.out + lj);
      }
      if (!((pw >> (lj % 32)) & 1)) break;  // final: the root
      cur = t;
      t = nt;
      // every hop is written back: walkers through this word jump to where
      // this walk has got (concurrent pointer doubling)
      if (kSingle) st_relaxed_u64(me.out + li, t);
      else st_relaxed_sys_u64(me.out + li, t);
    }
    if (err) record_error(ctx, DERR_CORRUPT);
  }
}

// Pending words take their root's value (roots are never pending, so nothing
// read here is being written). mode 2: every pending word (its pointer is its
// root after the walks of modes 0 and 1); then each bitmap word is cleared.
// Single view, chain nodes walked by mode 0 only: mode 0 gathers the other
// pending words (leaves) through their chain node — the leaf points at a chain
// node (marked by the decoder) or at a final word, and the chain node at its
// root — and writes only leaves; mode 1 then gathers the chain nodes and
// clears the bitmaps.
__global__ void __launch_bounds__(256) dp_gather_roots_kernel(const __grid_constant__ DpViews V,
                                                             const uint8_t* stream, uint64_t w_lo, uint64_t w_hi,
                                                             LaunchCtx ctx, const uint32_t* any_pend, int mode) {
  if (any_pend && *any_pend != ctx.epoch) return;
  const DpView& me = V.v[V.self];
  const uint64_t hi = dp_hi(V, stream, w_hi);
  const uint32_t lane = threadIdx.x & 31;
  const bool clear = mode != 0;
  for (uint64_t base = w_lo + (blockIdx.x * 256ull + threadIdx.x - lane); base < hi; base += gridDim.x * 256ull) {
    uint32_t bits = __ldcg(me.pend + base / 32);
    if (!bits) {  // warp-uniform; a chain node that is not pending may still be marked
      if (clear && lane == 0) me.tgt[base / 32] = 0;
      continue;
    }
    if (mode != 2) {
      const uint32_t nodes = __ldcg(me.tgt + base / 32);
      bits &= mode == 1 ? nodes : ~nodes;
    }
    const uint64_t li = base + lane;
    if (((bits >> lane) & 1) && li < hi) {
      uint64_t r = __ldcg(me.out + li);
      if (mode == 0 && r < me.first + li && r >= me.first) {  // a leaf: through its chain node
        const uint64_t lr = r - me.first;
        if ((__ldcg(me.pend + lr / 32) >> (lr % 32)) & 1) r = __ldcg(me.out + lr);
      }
      const DpView& w = V.v[dp_owner(V, r)];
      if (r >= me.first + li || r < w.first || r - w.first >= w.n) record_error(ctx, DERR_CORRUPT);
      else me.out[li] = ld_relaxed_sys_u64(w.out + (r - w.first));
    }
    if (clear) {
      __syncwarp();
      if (lane == 0) {
        me.pend[base / 32] = 0;
        me.tgt[base / 32] = 0;
      }
    }
  }
}

// The chain-node list of a single-view decode: the walk runs over the list
// (a few percent of the pending words on repeat-heavy data) instead of
// scanning every bitmap word, in list order (≈ index order: tiles append as
// they are decoded), writing back every hop.
#ifndef LCF_WALK_U
#define LCF_WALK_U 2
#endif
constexpr int kWalkU = LCF_WALK_U;  // list entries walked together per thread (their hops overlap)
__global__ void __launch_bounds__(256) dp_walk_nodes_kernel(DpView me, const uint32_t* __restrict__ nodes,
                                                           const uint32_t* __restrict__ n_nodes, uint64_t cap,
                                                           LaunchCtx ctx, const uint32_t* any_pend) {
  if (any_pend && *any_pend != ctx.epoch) return;
  const uint64_t cnt = umin64(*n_nodes, cap);
  const uint64_t stride = (uint64_t)gridDim.x * 256;
  for (uint64_t k0 = blockIdx.x * 256ull + threadIdx.x; k0 < cnt; k0 += stride * kWalkU) {
    uint64_t c[kWalkU], cur[kWalkU], t[kWalkU];
    bool on[kWalkU];
#pragma unroll
    for (int u = 0; u < kWalkU; ++u) {
      const uint64_t k = k0 + stride * u;
      c[u] = k < cnt ? nodes[k] : ~0ull;
      on[u] = c[u] < me.n && ((__ldcg(me.pend + c[u] / 32) >> (c[u] % 32)) & 1);  // (a final word: nothing)
      cur[u] = c[u];
      t[u] = on[u] ? __ldcg(me.out + c[u]) : 0ull;
    }
    bool any = false;
#pragma unroll
    for (int u = 0; u < kWalkU; ++u) any |= on[u];
    while (any) {
      uint32_t pw[kWalkU];
      uint64_t nt[kWalkU];
#pragma unroll
      for (int u = 0; u < kWalkU; ++u) {
        if (on[u] && t[u] >= cur[u]) {  // chains point strictly backwards
          record_error(ctx, DERR_CORRUPT);
          on[u] = false;
        }
        // the bit and the word are fetched together (one round trip per hop)
        pw[u] = on[u] ? __ldcg(me.pend + t[u] / 32) : 0u;
        nt[u] = on[u] ? ld_relaxed_u64(me.out + t[u]) : 0ull;
      }
      any = false;
#pragma unroll
      for (int u = 0; u < kWalkU; ++u) {
        if (!on[u]) continue;
        if (!((pw[u] >> (t[u] % 32)) & 1)) {  // t is final: the root (already stored)
          on[u] = false;
          continue;
        }
        cur[u] = t[u];
        t[u] = nt[u];
        st_relaxed_u64(me.out + c[u], t[u]);  // every hop is written back (concurrent pointer doubling)
        any = true;
      }
    }
  }
}

__global__ void __launch_bounds__(256) dp_gather_nodes_kernel(DpView me, const uint32_t* __restrict__ nodes,
                                                             const uint32_t* __restrict__ n_nodes, uint64_t cap,
                                                             LaunchCtx ctx, const uint32_t* any_pend) {
  if (any_pend && *any_pend != ctx.epoch) return;
  const uint64_t cnt = umin64(*n_nodes, cap);
  for (uint64_t k = blockIdx.x * 256ull + threadIdx.x; k < cnt; k += (uint64_t)gridDim.x * 256) {
    const uint64_t c = nodes[k];
    if (c >= me.n || !((__ldcg(me.pend + c / 32) >> (c % 32)) & 1)) continue;
    const uint64_t r = __ldcg(me.out + c);
    if (r >= c) record_error(ctx, DERR_CORRUPT);
    else me.out[c] = __ldcg(me.out + r);
  }
}

// The leaves of a single-view decode (pending words that are not chain
// nodes), after the chain nodes' walk: each takes its value through its chain
// node (or straight from a final target). A warp takes kLeafU bitmap words at
// a time so that the five dependent loads of every leaf overlap with those of
// the others (the pass is latency-bound on L2 round trips).
#ifndef LCF_LEAF_U
#define LCF_LEAF_U 4
#endif
constexpr int kLeafU = LCF_LEAF_U;
__global__ void __launch_bounds__(256) dp_gather_leaves_kernel(DpView me, const uint8_t* stream, uint64_t w_lo,
                                                              uint64_t w_hi, LaunchCtx ctx, const uint32_t* any_pend) {
  if (any_pend && *any_pend != ctx.epoch) return;
  uint64_t hi = w_hi < me.n ? w_hi : me.n;
  if (stream) {
    const uint64_t nw = reinterpret_cast<const uint64_t*>(stream)[1] / 8;
    hi = hi < nw ? hi : nw;
  }
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t wg = (blockIdx.x * 256ull + threadIdx.x) >> 5, nwarps = gridDim.x * 8ull;
  for (uint64_t base = w_lo + wg * 32 * kLeafU; base < hi; base += nwarps * 32 * kLeafU) {
    uint32_t bits[kLeafU];
#pragma unroll
    for (int u = 0; u < kLeafU; ++u) {
      const uint64_t b = base + 32 * u;
      bits[u] = b < hi ? __ldcg(me.pend + b / 32) & ~__ldcg(me.tgt + b / 32) : 0u;
    }
    uint64_t r[kLeafU];
    bool act[kLeafU];
#pragma unroll
    for (int u = 0; u < kLeafU; ++u) {
      const uint64_t li = base + 32 * u + lane;
      act[u] = ((bits[u] >> lane) & 1) && li < hi;
      r[u] = act[u] ? __ldcg(me.out + li) : 0ull;
    }
    uint32_t pr[kLeafU];
#pragma unroll
    for (int u = 0; u < kLeafU; ++u) {
      const uint64_t li = base + 32 * u + lane;
      if (act[u] && r[u] >= li) {  // chains point backwards
        record_error(ctx, DERR_CORRUPT);
        act[u] = false;
      }
      pr[u] = act[u] ? __ldcg(me.pend + r[u] / 32) : 0u;
    }
#pragma unroll
    for (int u = 0; u < kLeafU; ++u)
      if (act[u] && ((pr[u] >> (r[u] % 32)) & 1)) r[u] = __ldcg(me.out + r[u]);  // the chain node's root
    uint64_t v[kLeafU];
#pragma unroll
    for (int u = 0; u < kLeafU; ++u) {
      if (act[u] && r[u] >= me.n) {
        record_error(ctx, DERR_CORRUPT);
        act[u] = false;
      }
      v[u] = act[u] ? __ldcg(me.out + r[u]) : 0ull;
    }
#pragma unroll
    for (int u = 0; u < kLeafU; ++u)
      if (act[u]) me.out[base + 32 * u + lane] = v[u];
  }
}

int roots_grid(const void* kern, uint64_t words) {
  const uint64_t cap = (uint64_t)resident_capacity(kern, 256, 0);
  const uint64_t need = (words + 255) / 256;
  return (int)(need < cap ? (need ? need : 1) : cap);
}
}  // namespace

void launch_dp_find_roots(const DpViews& v, const uint8_t* stream, uint64_t w_lo, uint64_t w_hi,
                          const LaunchCtx& ctx, const uint32_t* any_pend, cudaStream_t st, int mode) {
  if (w_hi <= w_lo) return;
  KTrace kt("dp_find_roots", st);
  if (v.count == 1)
    dp_find_roots_kernel<true><<<roots_grid((const void*)dp_find_roots_kernel<true>, w_hi - w_lo), 256, 0, st>>>(
        v, stream, w_lo, w_hi, ctx, any_pend, mode);
  else
    dp_find_roots_kernel<false><<<roots_grid((const void*)dp_find_roots_kernel<false>, w_hi - w_lo), 256, 0, st>>>(
        v, stream, w_lo, w_hi, ctx, any_pend, mode);
}

void launch_dp_gather_leaves(const DpView& v, const uint8_t* stream, uint64_t w_lo, uint64_t w_hi,
                             const LaunchCtx& ctx, const uint32_t* any_pend, cudaStream_t st) {
  if (w_hi <= w_lo) return;
  KTrace kt("dp_gather_leaves", st);
  dp_gather_leaves_kernel<<<roots_grid((const void*)dp_gather_leaves_kernel, (w_hi - w_lo) / kLeafU), 256, 0, st>>>(
      v, stream, w_lo, w_hi, ctx, any_pend);
}

void launch_dp_nodes(const DpView& v, const uint32_t* nodes, const uint32_t* n_nodes, uint64_t cap,
                     const LaunchCtx& ctx, const uint32_t* any_pend, bool gather, cudaStream_t st) {
  if (!cap) return;
  if (gather) {
    KTrace kt("dp_gather_nodes", st);
    dp_gather_nodes_kernel<<<roots_grid((const void*)dp_gather_nodes_kernel, cap), 256, 0, st>>>(v, nodes, n_nodes, cap,
                                                                                               ctx, any_pend);
  } else {
    KTrace kt("dp_walk_nodes", st);
    dp_walk_nodes_kernel<<<roots_grid((const void*)dp_walk_nodes_kernel, cap), 256, 0, st>>>(v, nodes, n_nodes, cap,
                                                                                           ctx, any_pend);
  }
}

void launch_dp_gather_roots(const DpViews& v, const uint8_t* stream, uint64_t w_lo, uint64_t w_hi,
                            const LaunchCtx& ctx, const uint32_t* any_pend, cudaStream_t st, int mode) {
  if (w_hi <= w_lo) return;
  KTrace kt(mode == 0 ? "dp_gather_leaves" : "dp_gather_roots", st);
  dp_gather_roots_kernel<<<roots_grid((const void*)dp_gather_roots_kernel, w_hi - w_lo), 256, 0, st>>>(
      v, stream, w_lo, w_hi, ctx, any_pend, mode);
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
