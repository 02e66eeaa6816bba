// lcf_fcm.cu — the FCM distance array of DPratio (§3.4) on
// sm_100a, without a library sort.
//
// L172–176: hash the three preceding words of every position i, sort the
// pairs (h, i), and find for i the nearest of the (up to) four preceding pairs
// in sorted order with the same hash whose word equals x[i]; dist[i] = i − j.
//
// The (h, i) order is produced by a two-pass stable LSD radix sort over the two
// 10-bit digits of the 20-bit hash. Pass 1 reads x itself (the hash is computed
// on the fly from a warp's 32 consecutive words plus three carried words), so
// there is no separate hash array. A sort record is one u64:
//     h (20 bits) | fp (12-bit fingerprint of x[i]) | i (32 bits)
// and the match kernel gathers x only where fingerprints agree.
//
// Each pass is three kernels over tiles of kTile = 16 Ki records, 16 warps per
// tile, warp w owning records [w·1024, (w+1)·1024) of the tile:
//   sort_hist    per-tile digit counts (shared atomics)
//   sort_scan    per-digit exclusive prefix over tiles (column scan) + totals
//   sort_scatter in rounds of 8 Ki records: per-warp digit counts → per-warp
//                stage slots inside the round's digit runs; each warp ranks
//                equal digits in lane order (a tag store per digit detects
//                clashes, five ballots on the winning lane id match the peers)
//                → the round's records sorted in a shared stage → copied out
//                with each digit run contiguous
// (LCF_ONESWEEP builds a measured-slower onesweep variant: below.)
#include "lcf_fcm.cuh"
#include "lcf_kernels.cuh"
#include "lcf_pipe.cuh"

namespace lcf {
namespace {

using fcm::hi_mul;
using fcm::kRecFpShift;
using fcm::kRecHashShift;
using fcm::kRecIdxMask;
constexpr uint64_t FCM_K1 = fcm::K1, FCM_K2 = fcm::K2, FCM_K3 = fcm::K3;
constexpr int kDigitBits = 10, kDigits = 1 << kDigitBits;
#ifndef LCF_WARP_RECS
#define LCF_WARP_RECS 1024
#endif
constexpr int kSortWarps = 16, kSortThreads = kSortWarps * 32, kWarpRecs = LCF_WARP_RECS;
constexpr uint32_t kTile = kSortWarps * kWarpRecs;
constexpr uint32_t kNoDigit = kDigits;  // records past n
constexpr int kMatchBlock = 256;
constexpr int kScanWarps = 32, kScanBlocks = kDigits / 8;  // 8 digits per CTA (sort_scan_kernel)

__device__ __forceinline__ uint32_t rec_digit(uint64_t rec, int pass) {
  return pass == 0 ? (uint32_t)(rec >> kRecHashShift) & (kDigits - 1) : (uint32_t)(rec >> (kRecHashShift + kDigitBits));
}

// Record from x[i] and the high words of the three hash products (only bits
// 44..63 of the 64-bit hash value are kept: bits 12..31 of its high word).
__device__ __forceinline__ uint64_t make_rec(uint64_t xi, uint32_t hw, uint64_t i) {
  const uint64_t h = hw >> 12;  // 20-bit hash (A-14)
  const uint32_t f = (uint32_t)(xi ^ (xi >> 32));
  const uint32_t fp = (f ^ (f >> 12) ^ (f >> 24)) & 0xFFFu;
  return (h << kRecHashShift) | ((uint64_t)fp << kRecFpShift) | i;
}

// Lanes whose winner id (5 bits) equals this lane's (valid lanes only).
__device__ __forceinline__ uint32_t winner_peers(uint32_t win, bool valid) {
  uint32_t peers = __ballot_sync(0xFFFFFFFFu, valid);
#pragma unroll
  for (int b = 0; b < 5; ++b) {
    const bool bit = (win >> b) & 1;
    const uint32_t bb = __ballot_sync(0xFFFFFFFFu, bit);
    peers &= bit ? bb : ~bb;
  }
  return peers;
}

// The records of one warp's range in index order, kBatch·32 at a time: all
// loads of a batch are issued before any record is formed (memory-level
// parallelism). Pass 0 builds records from x: lane l computes the products
// x[i]·K1, x[i]·K2, x[i]·K3 of its own word and the hash of position i takes
// them from lanes l−1, l−2, l−3 (one 32-bit rotation shuffle each); lanes
// 0..2 use the rotated values of the previous group. Pass 1 reads the
// records of pass 0.
#ifndef LCF_HIST_BATCH
#define LCF_HIST_BATCH 8  // 4: 2×70.0 us, 8: 2×71.2, 16: 2×85.6, 32: 2×82.9 (Miranda)
#endif
constexpr int kBatch = LCF_HIST_BATCH;  // records per lane per load batch (histogram kernel)
template <int PASS, int B = kBatch>
struct RecReader {
  const uint64_t* src;
  uint64_t n, i0;
  uint32_t r1p, r2p, r3p;  // previous group's rotated product words (pass 0)
  uint64_t v[B];
  // halo: words src[−halo … −1] precede the array (a shard's context, ≤ 3)
  __device__ __forceinline__ RecReader(const uint64_t* s, uint64_t n_, uint64_t start, uint32_t lane,
                                       uint32_t halo = 0)
      : src(s), n(n_), i0(start) {
    if (PASS == 0) {  // the group before `start`: only its lanes 29..31 matter
      const int64_t j = (int64_t)start - 32 + (int64_t)lane;
      const uint64_t y = (lane >= 29 && j >= -(int64_t)halo && (j < 0 || (uint64_t)j < n)) ? src[j] : 0;
      rotate(y, lane, r1p, r2p, r3p);
    }
  }
  __device__ __forceinline__ static void rotate(uint64_t y, uint32_t lane, uint32_t& r1, uint32_t& r2,
                                                uint32_t& r3) {
    r1 = __shfl_sync(0xFFFFFFFFu, hi_mul(y, FCM_K1), (lane + 31) & 31);
    r2 = __shfl_sync(0xFFFFFFFFu, hi_mul(y, FCM_K2), (lane + 30) & 31);
    r3 = __shfl_sync(0xFFFFFFFFu, hi_mul(y, FCM_K3), (lane + 29) & 31);
  }
  __device__ __forceinline__ void load(uint32_t lane) {
#pragma unroll
    for (int k = 0; k < B; ++k) {
      const uint64_t i = i0 + 32 * k + lane;
      v[k] = i < n ? src[i] : 0;
    }
  }
  // record of group k of the loaded batch (index i0 + 32k + lane)
  __device__ __forceinline__ uint64_t rec(int k, uint32_t lane, bool& valid) {
    const uint64_t i = i0 + 32 * k + lane;
    valid = i < n;
    if (PASS == 1) return v[k];
    uint32_t r1, r2, r3;
    rotate(v[k], lane, r1, r2, r3);
    const uint32_t a1 = lane >= 1 ? r1 : r1p, a2 = lane >= 2 ? r2 : r2p, a3 = lane >= 3 ? r3 : r3p;
    r1p = r1;
    r2p = r2;
    r3p = r3;
    return make_rec(v[k], a1 ^ a2 ^ a3, i);
  }
  __device__ __forceinline__ void advance() { i0 += 32 * B; }
};

template <int PASS>
__global__ void __launch_bounds__(kSortThreads) sort_hist_kernel(const uint64_t* __restrict__ src, uint64_t n,
                                                                 uint32_t* __restrict__ counts, uint32_t halo) {
  __shared__ uint32_t hist[kDigits];
  const uint32_t warp = warp_index_uniform(), lane = threadIdx.x & 31;
  for (uint32_t d = threadIdx.x; d < kDigits; d += kSortThreads) hist[d] = 0;
  __syncthreads();
  const uint64_t start = (uint64_t)blockIdx.x * kTile + warp * kWarpRecs;
  RecReader<PASS> rd(src, n, start, lane, halo);
  for (int s = 0; s < kWarpRecs / (32 * kBatch); ++s, rd.advance()) {
    if (rd.i0 >= n) break;  // warp-uniform
    rd.load(lane);
#pragma unroll
    for (int k = 0; k < kBatch; ++k) {
      bool valid;
      const uint64_t rec = rd.rec(k, lane, valid);
      const uint32_t d = valid ? rec_digit(rec, PASS) : kNoDigit;
      if (valid) atomicAdd(&hist[d], 1u);
    }
  }
  __syncthreads();
  for (uint32_t d = threadIdx.x; d < kDigits; d += kSortThreads) counts[(uint64_t)blockIdx.x * kDigits + d] = hist[d];
}

// counts[t][d] → exclusive prefix over tiles t of digit d; tot[d] = total.
// A CTA owns kScanDig digits (one 32-byte sector of a count row); lane l
// reads digit l mod kScanDig of tile t0 + 4k + l / kScanDig, so a warp covers
// four consecutive rows per load and 128 CTAs share the matrix.
constexpr int kScanDig = 8, kScanSub = 32 / kScanDig;
__global__ void __launch_bounds__(kScanWarps * 32) sort_scan_kernel(uint32_t* __restrict__ counts, uint32_t n_tiles,
                                                                   uint32_t* __restrict__ tot) {
  __shared__ uint32_t part[kScanWarps][32];
  const uint32_t warp = warp_index_uniform(), lane = threadIdx.x & 31;
  const uint32_t dl = lane % kScanDig, sub = lane / kScanDig;
  const uint32_t d = blockIdx.x * kScanDig + dl;
  const uint32_t t0 = (uint32_t)((uint64_t)warp * n_tiles / kScanWarps);
  const uint32_t t1 = (uint32_t)((uint64_t)(warp + 1) * n_tiles / kScanWarps);
  uint32_t s = 0;
#pragma unroll 4
  for (uint32_t t = t0 + sub; t < t1; t += kScanSub) s += counts[(uint64_t)t * kDigits + d];
  // this digit's sum over the warp's rows: combine the kScanSub row phases
#pragma unroll
  for (int k = kScanDig; k < 32; k <<= 1) s += __shfl_xor_sync(0xFFFFFFFFu, s, k);
  part[warp][lane] = s;
  __syncthreads();
  uint32_t run = 0;
  for (uint32_t w = 0; w < warp; ++w) run += part[w][dl];
  if (warp == kScanWarps - 1 && sub == 0) tot[d] = run + s;
  constexpr int kB = 4;  // row groups loaded before any is rewritten
  for (uint32_t t = t0; t < t1; t += kScanSub * kB) {
    uint32_t v[kB];
#pragma unroll
    for (int b = 0; b < kB; ++b) {
      const uint32_t tt = t + b * kScanSub + sub;
      v[b] = tt < t1 ? counts[(uint64_t)tt * kDigits + d] : 0u;
    }
#pragma unroll
    for (int b = 0; b < kB; ++b) {
      const uint32_t tt = t + b * kScanSub + sub;
      uint32_t incl = v[b];  // prefix over the kScanSub consecutive rows of this load
#pragma unroll
      for (int k = kScanDig; k < 32; k <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, k);
        if ((int)lane >= k) incl += y;
      }
      if (tt < t1) counts[(uint64_t)tt * kDigits + d] = run + incl - v[b];
      run += __shfl_sync(0xFFFFFFFFu, incl, 32 - kScanDig + dl);
    }
  }
}

// Stable scatter of one tile, in kRounds rounds of kRound records; in round r
// warp w owns records [r·kRound + w·256, +256) of the tile (8 groups of 32, one
// register batch), so round, warp, group and lane order is index order.
//   1. per-warp digit counts (packed u16 pairs, shared atomics)
//   2. per digit: exclusive prefix over the warps; the round's digit starts
//   3. rank inside the warp (ballot-matched equal digits, lane order) and put
//      the record at its sorted place in the round's shared stage
//   4. copy the stage out: record j of digit d goes to run[d] + j − start[d],
//      so consecutive threads write consecutive positions of a digit run
#ifndef LCF_SCAT_WARPS
#define LCF_SCAT_WARPS 16
#endif
#ifndef LCF_SCAT_BATCH
#define LCF_SCAT_BATCH 16  // 8192-record rounds, 1 CTA/SM: 2×639→2×618 us (8: 2 CTAs/SM; 32: spills;
                           // 32 warps × 8: 2×624 us)
#endif
#ifndef LCF_SCAT_MINB
#define LCF_SCAT_MINB 1
#endif
#ifndef LCF_SCAT_PREFETCH
#define LCF_SCAT_PREFETCH 1
#endif
constexpr int kSW = LCF_SCAT_WARPS, kST = kSW * 32, kSB = LCF_SCAT_BATCH;
constexpr int kRound = kST * kSB;  // records per round
// digit pairs per owning thread; with 1024 threads only the first 512 own a pair
constexpr int kP = kDigits / 2 / kST > 0 ? kDigits / 2 / kST : 1;
constexpr int kOwners = kDigits / 2 / kP;
static_assert(kP * 2 * kOwners == kDigits && kOwners <= kST, "digit pairs divide over the threads");
constexpr int kRounds = kTile / kRound;
static_assert(kRounds * kRound == kTile, "tile = whole rounds");
// LCF_SCAT_U32: one u32 count per (warp, digit) instead of packed u16 pairs —
// then lanes of distinct digits never share a word, and the rank update is a
// plain store by each digit's leader instead of a shared atomic
#ifndef LCF_SCAT_U32
#define LCF_SCAT_U32 1
#endif
struct ScatterSmem {
  uint64_t stage[kRound];
#if LCF_SCAT_U32
  uint32_t wcnt[kSW][kDigits];      // count, then the warp's next stage slot, per digit
#else
  uint32_t wcnt[kSW][kDigits / 2];  // packed u16 pair per word
#endif
  uint32_t run[kDigits];                   // next output position of each digit (tile-wide)
  uint32_t rstart[kDigits];                // round: first stage slot of each digit
  uint32_t delta[kDigits];                 // round: output position − stage slot of each digit
#if LCF_SCAT_U32
  uint32_t rtot[kDigits];                  // round: digit totals
#else
  uint32_t rtot[kDigits / 2];              // round: packed digit totals
#endif
  uint32_t wsum[kSW];
  uint8_t tag[kSW][kDigits];        // per warp: last lane that claimed a digit
};

template <int PASS>
__global__ void __launch_bounds__(kST, LCF_SCAT_MINB) sort_scatter_kernel(const uint64_t* __restrict__ src, uint64_t n,
                                                                    const uint32_t* __restrict__ offs,
                                                                    const uint32_t* __restrict__ tot,
                                                                    uint64_t* __restrict__ dst, uint32_t halo) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  ScatterSmem& S = *reinterpret_cast<ScatterSmem*>(smem_raw);
  const uint32_t tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const uint32_t lt = (1u << lane) - 1u;
  // Thread tid owns the kP digit pairs [kP·tid, kP·tid + kP), i.e. digits
  // [2kP·tid, 2kP·tid + 2kP). Block exclusive scan of per-digit values c[]
  // (in this thread's digit order) → ex[] (contains a __syncthreads).
  const bool owner = tid < (uint32_t)kOwners;
  auto digit_scan = [&](const uint32_t (&c)[2 * kP], uint32_t (&ex)[2 * kP]) {
    uint32_t own = 0;
#pragma unroll
    for (int j = 0; j < 2 * kP; ++j) own += c[j];
    uint32_t x = own;
#pragma unroll
    for (int k = 1; k < 32; k <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, k);
      if ((int)lane >= k) x += y;
    }
    if (lane == 31) S.wsum[warp] = x;
    __syncthreads();
    uint32_t base = x - own;
    for (uint32_t w = 0; w < warp; ++w) base += S.wsum[w];
#pragma unroll
    for (int j = 0; j < 2 * kP; ++j) {
      ex[j] = base;
      base += c[j];
    }
  };
  {  // digit bases (exclusive scan of tot) + this tile's offsets
    uint32_t c[2 * kP], ex[2 * kP];
#pragma unroll
    for (int j = 0; j < 2 * kP; ++j) c[j] = owner ? tot[2 * kP * tid + j] : 0u;
    digit_scan(c, ex);
    const uint32_t* o = offs + (uint64_t)blockIdx.x * kDigits;
    if (owner)
#pragma unroll
      for (int j = 0; j < 2 * kP; ++j) S.run[2 * kP * tid + j] = ex[j] + o[2 * kP * tid + j];
  }
  const uint64_t tile0 = (uint64_t)blockIdx.x * kTile;
  // the next round's loads are issued before this round's copy-out (step 4)
  RecReader<PASS, kSB> rd(src, n, tile0 + warp * 32 * kSB, lane, halo);
  rd.load(lane);
  for (int r = 0; r < kRounds; ++r) {
    const uint64_t r0 = tile0 + (uint64_t)r * kRound;
    if (r0 >= n) break;  // block-uniform
    const uint32_t nr = (uint32_t)umin64(kRound, n - r0);
    if (!LCF_SCAT_PREFETCH && r > 0) {
      rd = RecReader<PASS, kSB>(src, n, r0 + warp * 32 * kSB, lane, halo);
      rd.load(lane);
    }
    // 1. this warp's records of the round and its digit counts
#pragma unroll
#if LCF_SCAT_U32
    for (int j = lane; j < kDigits; j += 32) S.wcnt[warp][j] = 0;
#else
    for (int j = lane; j < kDigits / 2; j += 32) S.wcnt[warp][j] = 0;
#endif
    __syncwarp();
    uint64_t rec[kSB];
    uint32_t dg[kSB];
    bool ok[kSB];
#pragma unroll
    for (int k = 0; k < kSB; ++k) {
      rec[k] = rd.rec(k, lane, ok[k]);
      dg[k] = ok[k] ? rec_digit(rec[k], PASS) : 0u;
#if LCF_SCAT_U32
      if (ok[k]) atomicAdd(&S.wcnt[warp][dg[k]], 1u);
#else
      if (ok[k]) atomicAdd(&S.wcnt[warp][dg[k] >> 1], 1u << (16 * (dg[k] & 1)));
#endif
    }
    __syncthreads();
    // 2. this thread's digit pairs: prefix over the warps (packed: sums ≤ kRound per half)
#if LCF_SCAT_U32
    {
      uint32_t c[2 * kP], ex[2 * kP];
#pragma unroll
      for (int j = 0; j < 2 * kP; ++j) {
        const uint32_t dj = 2 * kP * tid + j;
        uint32_t tw = 0;
        if (owner) {
#pragma unroll
          for (int w = 0; w < kSW; ++w) {
            const uint32_t v = S.wcnt[w][dj];
            S.wcnt[w][dj] = tw;
            tw += v;
          }
        }
        c[j] = tw;
      }
      digit_scan(c, ex);
      if (owner)
#pragma unroll
        for (int j = 0; j < 2 * kP; ++j) {
          const uint32_t dj = 2 * kP * tid + j;
#pragma unroll
          for (int w = 0; w < kSW; ++w) S.wcnt[w][dj] += ex[j];  // absolute stage slots
          S.delta[dj] = S.run[dj] - ex[j];
          S.rtot[dj] = c[j];
        }
    }
#else
    {
      uint32_t c[2 * kP], ex[2 * kP];
#pragma unroll
      for (int q = 0; q < kP; ++q) {
        const uint32_t pq = kP * tid + q;
        uint32_t tw = 0;
        if (owner) {
#pragma unroll
          for (int w = 0; w < kSW; ++w) {
            const uint32_t v = S.wcnt[w][pq];
            S.wcnt[w][pq] = tw;
            tw += v;
          }
          S.rtot[pq] = tw;
        }
        c[2 * q] = tw & 0xFFFFu;
        c[2 * q + 1] = tw >> 16;
      }
      digit_scan(c, ex);  // (its barrier also publishes wcnt)
      if (owner)
#pragma unroll
        for (int j = 0; j < 2 * kP; ++j) {
          S.rstart[2 * kP * tid + j] = ex[j];
          S.delta[2 * kP * tid + j] = S.run[2 * kP * tid + j] - ex[j];
        }
    }
#endif
    __syncthreads();
    // 3. ranks → stage
#pragma unroll
    for (int k = 0; k < kSB; ++k) {
      const uint32_t d = dg[k];
      // equal digits inside the group are detected through a tag per digit
      // (one of the lanes that share a digit wins the byte store, the others
      // read another lane id back); only then are the peers matched exactly
      if (ok[k]) S.tag[warp][d] = (uint8_t)lane;
      __syncwarp();
      // every lane of a digit reads back the same winning lane id, and lanes of
      // different digits read different ids (a lane has one digit): the peers
      // are the lanes with my winner — five ballots on its bits instead of ten
      // on the digit's
      const uint32_t win = S.tag[warp][d];
      const bool clash = __any_sync(0xFFFFFFFFu, ok[k] && win != lane);
      const uint32_t peers = clash ? winner_peers(win, ok[k]) : (1u << lane);
#if LCF_SCAT_U32
      uint32_t* wc = &S.wcnt[warp][d];
      const uint32_t slot = ok[k] ? *wc : 0u;  // this warp's next stage slot of digit d
      __syncwarp();
      if (ok[k]) {
        S.stage[slot + __popc(peers & lt)] = rec[k];
        if (lane == (uint32_t)__ffs(peers) - 1) *wc = slot + __popc(peers);  // one writer per digit
      }
#else
      uint32_t* wc = &S.wcnt[warp][d >> 1];
      const uint32_t sh = 16 * (d & 1);
      const uint32_t rbase = ok[k] ? (*wc >> sh) & 0xFFFFu : 0u;
      __syncwarp();
      if (ok[k]) {
        S.stage[S.rstart[d] + rbase + __popc(peers & lt)] = rec[k];
        if (lane == (uint32_t)__ffs(peers) - 1) atomicAdd(wc, (uint32_t)__popc(peers) << sh);
      }
#endif
      __syncwarp();
    }
    if (LCF_SCAT_PREFETCH && r + 1 < kRounds) {
      rd = RecReader<PASS, kSB>(src, n, r0 + kRound + warp * 32 * kSB, lane, halo);
      rd.load(lane);
    }
    __syncthreads();
    // 4. stage → dst, digit runs contiguous
    for (uint32_t j = tid; j < nr; j += kST) {
      const uint64_t v = S.stage[j];
      dst[S.delta[rec_digit(v, PASS)] + j] = v;
    }
    __syncthreads();
    if (owner) {
#if LCF_SCAT_U32
#pragma unroll
      for (int j = 0; j < 2 * kP; ++j) S.run[2 * kP * tid + j] += S.rtot[2 * kP * tid + j];
#else
#pragma unroll
      for (int q = 0; q < kP; ++q) {
        const uint32_t pq = kP * tid + q, t2 = S.rtot[pq];
        S.run[2 * pq] += t2 & 0xFFFFu;
        S.run[2 * pq + 1] += t2 >> 16;
      }
#endif
    }
    // (the next round's first barrier orders these updates before step 4)
  }
}

// ---- onesweep sort (LCF_ONESWEEP) ----------------------------------------------
// The global digit totals of BOTH passes come from one read of x
// (sort_ghist); each pass is then one kernel (sort_onesweep): persistent CTAs
// take tiles of kRound records by ticket, count the tile's digits, publish the
// counts, and find the tile's offset inside every digit run by a decoupled
// look-back over the earlier tiles' status words — no per-tile count matrix,
// no column scan, and no second histogram pass over the pass-0 records.
// Status word of (tile, digit): 0 = not yet published, else (value + 1) with
// bit 31 set once value is the inclusive prefix over tiles 0..t (else value is
// the tile's own count). n < 2^31 keeps value + 1 below bit 31.
// Measured slower than the hist/scan/scatter passes and kept for A/B builds
// only: 94 µs + 2 × 350 µs against 2 × (71 + 15 + 284) µs on
// Miranda; without the look-back (wrong offsets, a timing bound) 2 × 277 µs —
// the 148 lock-stepped tiles of a wave resolve their inclusive prefixes in a
// cascade, ≈ 2.3 µs per 8 Ki-record tile.
#ifndef LCF_ONESWEEP
#define LCF_ONESWEEP 0
#endif
#ifndef LCF_SWEEP_LB
#define LCF_SWEEP_LB 32  // status words read per round trip of a look-back walk
#endif
constexpr uint32_t kIncl = 0x80000000u;
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// tot2[0][d], tot2[1][d]: how many records have digit d in pass 0 / pass 1
// (tot2 pre-zeroed). Warps take kWarpRecs-record ranges grid-stride.
__global__ void __launch_bounds__(kSortThreads) sort_ghist_kernel(const uint64_t* __restrict__ x, uint64_t n,
                                                                  uint32_t* __restrict__ tot2, uint32_t halo) {
  __shared__ uint32_t hist[2][kDigits];
  const uint32_t warp = warp_index_uniform(), lane = threadIdx.x & 31;
  for (uint32_t d = threadIdx.x; d < 2 * kDigits; d += kSortThreads) (&hist[0][0])[d] = 0;
  __syncthreads();
  const uint64_t ranges = (n + kWarpRecs - 1) / kWarpRecs;
  for (uint64_t g = (uint64_t)blockIdx.x * kSortWarps + warp; g < ranges; g += (uint64_t)gridDim.x * kSortWarps) {
    RecReader<0> rd(x, n, g * kWarpRecs, lane, halo);
    for (int s = 0; s < kWarpRecs / (32 * kBatch); ++s, rd.advance()) {
      if (rd.i0 >= n) break;  // warp-uniform
      rd.load(lane);
#pragma unroll
      for (int k = 0; k < kBatch; ++k) {
        bool valid;
        const uint64_t rec = rd.rec(k, lane, valid);
        if (valid) {
          atomicAdd(&hist[0][rec_digit(rec, 0)], 1u);
          atomicAdd(&hist[1][rec_digit(rec, 1)], 1u);
        }
      }
    }
  }
  __syncthreads();
  for (uint32_t d = threadIdx.x; d < 2 * kDigits; d += kSortThreads) {
    const uint32_t c = (&hist[0][0])[d];
    if (c) atomicAdd(tot2 + d, c);
  }
}

struct OnesweepSmem {
  uint64_t stage[kRound];
  uint32_t wcnt[kSW][kDigits];  // count, then the warp's next stage slot, per digit
  uint32_t gbase[kDigits];      // first output position of each digit (exclusive scan of the totals)
  uint32_t delta[kDigits];      // tile: output position − stage slot of each digit
  uint32_t wsum[kSW];
  uint32_t tile[2];             // tickets (current, next)
  uint8_t tag[kSW][kDigits];    // per warp: last lane that claimed a digit
};

// One LSD pass: records src[0, n) → dst, stable by digit PASS. tot: this
// pass's global digit totals; status: ceil(n / kRound) × kDigits words, zeroed;
// ticket: zeroed. Tiles are taken in ticket order and a tile only waits on
// earlier tiles, whose holders are running: no deadlock.
template <int PASS>
__global__ void __launch_bounds__(kST, 1) sort_onesweep_kernel(const uint64_t* __restrict__ src, uint64_t n,
                                                               const uint32_t* __restrict__ tot,
                                                               uint32_t* __restrict__ status,
                                                               uint32_t* __restrict__ ticket,
                                                               uint64_t* __restrict__ dst, uint32_t halo) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  OnesweepSmem& S = *reinterpret_cast<OnesweepSmem*>(smem_raw);
  const uint32_t tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const uint32_t lt = (1u << lane) - 1u;
  const bool owner = tid < (uint32_t)kOwners;  // thread owns digits [2kP·tid, 2kP·tid + 2kP)
  auto digit_scan = [&](const uint32_t (&c)[2 * kP], uint32_t (&ex)[2 * kP]) {
    uint32_t own = 0;
#pragma unroll
    for (int j = 0; j < 2 * kP; ++j) own += c[j];
    uint32_t x = own;
#pragma unroll
    for (int k = 1; k < 32; k <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, k);
      if ((int)lane >= k) x += y;
    }
    if (lane == 31) S.wsum[warp] = x;
    __syncthreads();
    uint32_t base = x - own;
    for (uint32_t w = 0; w < warp; ++w) base += S.wsum[w];
#pragma unroll
    for (int j = 0; j < 2 * kP; ++j) {
      ex[j] = base;
      base += c[j];
    }
  };
  {  // digit bases
    uint32_t c[2 * kP], ex[2 * kP];
#pragma unroll
    for (int j = 0; j < 2 * kP; ++j) c[j] = owner ? tot[2 * kP * tid + j] : 0u;
    digit_scan(c, ex);
    if (owner)
#pragma unroll
      for (int j = 0; j < 2 * kP; ++j) S.gbase[2 * kP * tid + j] = ex[j];
  }
  const uint32_t nT = (uint32_t)((n + kRound - 1) / kRound);
  if (tid == 0) S.tile[0] = atomicAdd(ticket, 1u);
  __syncthreads();  // (also orders wsum reuse)
  uint32_t t = S.tile[0];
  RecReader<PASS, kSB> rd(src, n, (uint64_t)t * kRound + warp * 32 * kSB, lane, halo);
  if (t < nT) rd.load(lane);
  for (uint32_t it = 0; t < nT; ++it) {
    const uint64_t r0 = (uint64_t)t * kRound;
    const uint32_t nr = (uint32_t)umin64(kRound, n - r0);
    // 1. this warp's records of the tile and its digit counts
    for (int j = lane; j < kDigits; j += 32) S.wcnt[warp][j] = 0;
    __syncwarp();
    uint64_t rec[kSB];
    uint32_t dg[kSB];
    bool ok[kSB];
#pragma unroll
    for (int k = 0; k < kSB; ++k) {
      rec[k] = rd.rec(k, lane, ok[k]);
      dg[k] = ok[k] ? rec_digit(rec[k], PASS) : 0u;
      if (ok[k]) atomicAdd(&S.wcnt[warp][dg[k]], 1u);
    }
    __syncthreads();
    // 2. per digit: prefix over the warps and the tile's count, published at
    // once (successors add it up in their look-back), then the stage slots
    uint32_t c[2 * kP], ex[2 * kP];
#pragma unroll
    for (int j = 0; j < 2 * kP; ++j) {
      const uint32_t dj = 2 * kP * tid + j;
      uint32_t tw = 0;
      if (owner) {
#pragma unroll
        for (int w = 0; w < kSW; ++w) {
          const uint32_t v = S.wcnt[w][dj];
          S.wcnt[w][dj] = tw;
          tw += v;
        }
        st_relaxed_u32(status + (uint64_t)t * kDigits + dj, (t == 0 ? kIncl : 0u) | (tw + 1));
      }
      c[j] = tw;
    }
    digit_scan(c, ex);
    if (owner)
#pragma unroll
      for (int j = 0; j < 2 * kP; ++j)
#pragma unroll
        for (int w = 0; w < kSW; ++w) S.wcnt[w][2 * kP * tid + j] += ex[j];  // absolute stage slots
    if (tid == 0) S.tile[(it + 1) & 1] = atomicAdd(ticket, 1u);  // the next tile, for the prefetch
    __syncthreads();
    // 3. ranks → stage (as sort_scatter_kernel); the tile's offsets in the
    // digit runs are not needed before step 4
#pragma unroll
    for (int k = 0; k < kSB; ++k) {
      const uint32_t d = dg[k];
      if (ok[k]) S.tag[warp][d] = (uint8_t)lane;
      __syncwarp();
      const uint32_t win = S.tag[warp][d];
      const bool clash = __any_sync(0xFFFFFFFFu, ok[k] && win != lane);
      const uint32_t peers = clash ? winner_peers(win, ok[k]) : (1u << lane);
      uint32_t* wc = &S.wcnt[warp][d];
      const uint32_t slot = ok[k] ? *wc : 0u;
      __syncwarp();
      if (ok[k]) {
        S.stage[slot + __popc(peers & lt)] = rec[k];
        if (lane == (uint32_t)__ffs(peers) - 1) *wc = slot + __popc(peers);
      }
      __syncwarp();
    }
    const uint32_t tn = S.tile[(it + 1) & 1];
    if (tn < nT) {  // the next tile's loads fly during the look-back and the copy-out
      rd = RecReader<PASS, kSB>(src, n, (uint64_t)tn * kRound + warp * 32 * kSB, lane, halo);
      rd.load(lane);
    }
    // 2b. look-back: the tile's offset in each digit run = the sum of the
    // earlier tiles' counts, down to the nearest inclusive prefix. The status
    // words of the previous tile for all of the thread's digits are read at
    // once (usually inclusive already: one L2 round trip); walking further
    // reads kLB tiles per round trip
#ifndef LCF_SWEEP_NOLB
#define LCF_SWEEP_NOLB 0  // timing experiment only: no look-back (wrong offsets)
#endif
    if (owner && LCF_SWEEP_NOLB) {
#pragma unroll
      for (int j = 0; j < 2 * kP; ++j) S.delta[2 * kP * tid + j] = S.gbase[2 * kP * tid + j] - ex[j];
    } else if (owner) {
      uint32_t v0[2 * kP];
      const uint32_t* sp = status + (uint64_t)(t > 0 ? t - 1 : 0) * kDigits + 2 * kP * tid;
#pragma unroll
      for (int j = 0; j < 2 * kP; ++j) v0[j] = t > 0 ? ld_relaxed_u32(sp + j) : (kIncl | 1u);
#pragma unroll
      for (int j = 0; j < 2 * kP; ++j) {
        const uint32_t dj = 2 * kP * tid + j;
        while (v0[j] == 0) v0[j] = ld_relaxed_u32(sp + j);
        uint32_t excl = (v0[j] & ~kIncl) - 1;
        if (!(v0[j] & kIncl)) {  // tile t − 1 not yet inclusive: walk on
          constexpr int kLB = LCF_SWEEP_LB;
          bool done = false;
          for (int64_t s0 = (int64_t)t - 2; !done; s0 -= kLB) {
            uint32_t v[kLB];
#pragma unroll
            for (int b = 0; b < kLB; ++b)
              v[b] = s0 - b >= 0 ? ld_relaxed_u32(status + (uint64_t)(s0 - b) * kDigits + dj) : (kIncl | 1u);
#pragma unroll
            for (int b = 0; b < kLB; ++b) {
              if (done) break;
              while (v[b] == 0) v[b] = ld_relaxed_u32(status + (uint64_t)(s0 - b) * kDigits + dj);
              excl += (v[b] & ~kIncl) - 1;
              done = (v[b] & kIncl) != 0;
            }
          }
        }
        if (t > 0) st_relaxed_u32(status + (uint64_t)t * kDigits + dj, kIncl | (excl + c[j] + 1));
        S.delta[dj] = S.gbase[dj] + excl - ex[j];
      }
    }
    __syncthreads();
    // 4. stage → dst, digit runs contiguous
    for (uint32_t j = tid; j < nr; j += kST) {
      const uint64_t v = S.stage[j];
      dst[S.delta[rec_digit(v, PASS)] + j] = v;
    }
    t = tn;
    // (step 1's barrier of the next tile orders these reads of stage / delta
    // before they are rewritten)
  }
}

// Thread t covers the kMatchItems sorted positions k = 8t … 8t+7; for each,
// the nearest of the records k−1 … k−4 with the same hash and an equal word is
// the match (L174, A-14, A-15). Records of one hash are contiguous, so the walk
// stops at the first other hash. The 12 records a thread needs come from six
// 16-byte loads (no shared memory, no barriers). The distance array is
// pre-zeroed; only matches are scattered.
#ifndef LCF_MATCH_SPLIT
#define LCF_MATCH_SPLIT 1
#endif
#ifndef LCF_MATCH_ITEMS
#define LCF_MATCH_ITEMS 8
#endif
constexpr int kMatchItems = LCF_MATCH_ITEMS;
// Sharded DPratio (NEXT-1): per hash, the last ≤ 4 records (nearest first) of
// the words before this shard — global index and word — merged from the
// lower shards' summaries. Candidates of a record are its local same-hash
// predecessors first (nearer), then these (L174, A-14).
struct FcmCarry {
  const uint8_t* cnt;    // [2^20]
  const uint32_t* idx;   // [2^20][4]
  const uint64_t* val;   // [2^20][4]
};
constexpr uint64_t kHashes = 1ull << 20;
__host__ __device__ constexpr size_t carry_bytes() { return kHashes * (1 + 4 * 4 + 4 * 8); }

// CARRY: a shard after the first (compiled separately: the carry test costs
// the unsharded match a third of its time)
template <bool CARRY>
__global__ void __launch_bounds__(kMatchBlock) fcm_match_kernel(const uint64_t* __restrict__ x, uint64_t n,
                                                                const uint64_t* __restrict__ rec,
                                                                uint32_t* __restrict__ dist, FcmCarry carry,
                                                                uint64_t gbase, uint32_t ilo, uint32_t ihi) {
  constexpr bool carry_on = CARRY;
  const uint64_t groups = (n + kMatchItems - 1) / kMatchItems;
  for (uint64_t g = blockIdx.x * (uint64_t)kMatchBlock + threadIdx.x; g < groups;
       g += (uint64_t)gridDim.x * kMatchBlock) {
    const uint64_t k0 = g * kMatchItems;
    uint64_t r[4 + kMatchItems];  // records k0−4 … k0+7 (0 outside [0, n): never read as predecessors)
    if (k0 + kMatchItems <= n) {
      const ulonglong2* p = reinterpret_cast<const ulonglong2*>(rec + k0);
#pragma unroll
      for (int q = 0; q < kMatchItems / 2; ++q) {
        const ulonglong2 v = p[q];
        r[4 + 2 * q] = v.x;
        r[5 + 2 * q] = v.y;
      }
    } else {
#pragma unroll
      for (int j = 0; j < kMatchItems; ++j) r[4 + j] = k0 + j < n ? rec[k0 + j] : 0;
    }
    if (k0 >= 4) {
      const ulonglong2* p = reinterpret_cast<const ulonglong2*>(rec + k0 - 4);
      const ulonglong2 v0 = p[0], v1 = p[1];
      r[0] = v0.x;
      r[1] = v0.y;
      r[2] = v1.x;
      r[3] = v1.y;
    } else {
      r[0] = r[1] = r[2] = r[3] = 0;
    }
    // the high word of a record is h(20) | fp(12): equal hash ⇔ (a ^ b) >> 12 == 0,
    // equal hash and fingerprint ⇔ a == b
    uint32_t hw[4 + kMatchItems];
#pragma unroll
    for (int t = 0; t < 4 + kMatchItems; ++t) hw[t] = (uint32_t)(r[t] >> 32);
#pragma unroll
    for (int j = 0; j < kMatchItems; ++j) {
      const uint64_t k = k0 + j;
      if (k >= n) break;
      const uint32_t hk = hw[4 + j];
      const bool start = k == 0 || ((hw[3 + j] ^ hk) >> 12);  // first of its hash run here
      if (start && !carry_on) continue;  // no candidate at all
      const uint64_t rk = r[4 + j];
      const uint32_t i = (uint32_t)(rk & kRecIdxMask);
      uint32_t d = 0, used = 0;
      uint64_t xi = 0;
      bool have = false;
      if constexpr (!CARRY) {
        // deferred (no gather of x here): the nearest candidate with the same
        // hash and fingerprint, flagged if another one follows in the window;
        // the DPratio encoder compares the words in index order (L2-near for
        // repeats a few rows apart) and falls back to fcm::match_one only when
        // the nearest fails and another candidate exists
#pragma unroll
        for (int back = 1; back <= 4; ++back) {  // nearest first (pinned by Fig. 6)
          if ((uint64_t)back > k) break;        // sorted position k has only k predecessors
          const uint32_t hb = hw[4 + j - back];
          if ((hb ^ hk) >> 12) break;  // left the hash's run
          if (hb == hk) {
            if (d) {
              d |= fcm::kMulti;
              break;
            }
            d = i - (uint32_t)(r[4 + j - back] & kRecIdxMask);
          }
        }
        if (d && i - ilo < ihi - ilo) dist[i] = d;  // (this launch's index range only)
      } else {
#pragma unroll
      for (int back = 1; back <= 4; ++back) {  // nearest first (pinned by Fig. 6)
        if ((uint64_t)back > k) break;        // sorted position k has only k predecessors
        const uint32_t hb = hw[4 + j - back];
        if ((hb ^ hk) >> 12) break;  // left the hash's run
        if (CARRY) ++used;
        if (hb == hk) {              // same hash and fingerprint
          const uint32_t jj = (uint32_t)(r[4 + j - back] & kRecIdxMask);
          if (!have) {
            xi = x[i];
            have = true;
          }
          if (x[jj] == xi) {
            d = i - jj;
            break;
          }
        }
      }
      if (CARRY && d == 0 && used < 4) {  // the remaining candidates precede the shard
        const uint32_t h = hk >> 12, cc = carry.cnt[h];
#pragma unroll
        for (uint32_t q = 0; q < 4; ++q) {
          if (q >= cc || q + used >= 4) break;
          if (!have) {
            xi = x[i];
            have = true;
          }
          if (carry.val[4 * h + q] == xi) {
            d = (uint32_t)(gbase + i - carry.idx[4 * h + q]);
            break;
          }
        }
      }
      if (d) dist[i] = d;
      }
    }
  }
}

// Summary of a shard (sorted records rec[0, n)): per hash, the last ≤ 4
// records of its run (nearest first) as global index and word.
__global__ void __launch_bounds__(256) fcm_summary_kernel(const uint64_t* __restrict__ x, uint64_t n,
                                                         const uint64_t* __restrict__ rec, uint64_t gbase,
                                                         uint8_t* __restrict__ cnt, uint32_t* __restrict__ idx,
                                                         uint64_t* __restrict__ val) {
  for (uint64_t k = blockIdx.x * 256ull + threadIdx.x; k < n; k += (uint64_t)gridDim.x * 256) {
    const uint64_t hk = rec[k] >> kRecHashShift;
    if (k + 1 < n && (rec[k + 1] >> kRecHashShift) == hk) continue;  // not the end of the run
    uint32_t c = 0;
    for (uint32_t q = 0; q < 4 && q <= k; ++q) {
      const uint64_t r = rec[k - q];
      if ((r >> kRecHashShift) != hk) break;
      const uint32_t i = (uint32_t)(r & kRecIdxMask);
      idx[4 * hk + q] = (uint32_t)(gbase + i);
      val[4 * hk + q] = x[i];
      ++c;
    }
    cnt[hk] = (uint8_t)c;
  }
}

// Carry of shard g: per hash, walk the summaries of shards g−1, g−2, … 0 and
// keep the first four entries (most recent first). The summaries are read
// through pointers (local, or peers' mapped by CUDA IPC): a hash whose four
// entries come from shard g−1 never touches the older summaries.
struct SumPtrs {
  const uint8_t* p[64];
};
__global__ void __launch_bounds__(256) fcm_carry_merge_kernel(const __grid_constant__ SumPtrs S, uint32_t count,
                                                             uint8_t* __restrict__ out) {
  const uint64_t h = blockIdx.x * 256ull + threadIdx.x;
  if (h >= kHashes) return;
  auto idx_of = [&](const uint8_t* b) { return reinterpret_cast<const uint32_t*>(b + kHashes); };
  auto val_of = [&](const uint8_t* b) { return reinterpret_cast<const uint64_t*>(b + kHashes * 17); };
  uint32_t m = 0;
  for (int32_t r = (int32_t)count - 1; r >= 0 && m < 4; --r) {
    const uint8_t* b = S.p[r];
    const uint32_t c = b[h];
    for (uint32_t q = 0; q < c && m < 4; ++q, ++m) {
      reinterpret_cast<uint32_t*>(out + kHashes)[4 * h + m] = idx_of(b)[4 * h + q];
      reinterpret_cast<uint64_t*>(out + kHashes * 17)[4 * h + m] = val_of(b)[4 * h + q];
    }
  }
  out[h] = (uint8_t)m;
}

// The deferred candidates of the match kernel (distance | fcm::kMulti), in
// index order: x[i] is read coalesced and x[i − d] is L2-near for repeats a
// few rows back (a gather in sorted order costs two random sectors per
// candidate). A failed nearest candidate with another one in its window falls
// back to the full match of that word (fcm::match_one, rare).
__global__ void __launch_bounds__(256) fcm_verify_kernel(const uint64_t* __restrict__ x, uint64_t n,
                                                        const uint64_t* __restrict__ rec, uint32_t* __restrict__ dist,
                                                        uint32_t halo) {
  const uint64_t q4 = (n + 3) / 4;
  for (uint64_t q = blockIdx.x * 256ull + threadIdx.x; q < q4; q += (uint64_t)gridDim.x * 256) {
    uint4 dv;
    if (4 * q + 4 <= n) {
      dv = __ldcs(reinterpret_cast<const uint4*>(dist) + q);
    } else {
      dv.x = dist[4 * q];
      dv.y = 4 * q + 1 < n ? dist[4 * q + 1] : 0u;
      dv.z = 4 * q + 2 < n ? dist[4 * q + 2] : 0u;
      dv.w = 4 * q + 3 < n ? dist[4 * q + 3] : 0u;
    }
    if (!(dv.x | dv.y | dv.z | dv.w)) continue;
    const uint32_t raw[4] = {dv.x, dv.y, dv.z, dv.w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (!raw[j]) continue;
      const uint64_t i = 4 * q + j;
      const uint32_t d = raw[j] & ~fcm::kMulti;
      uint32_t v = d <= i && x[i - d] == x[i] ? d : 0u;
      if (!v && (raw[j] & fcm::kMulti)) v = fcm::match_one(x, rec, n, (uint32_t)i, halo);
      if (v != raw[j]) dist[i] = v;
    }
  }
}

uint64_t n_tiles_of(uint64_t n) { return (n + kTile - 1) / kTile; }

}  // namespace

static uint64_t n_sweep_tiles_of(uint64_t n) { return (n + kRound - 1) / kRound; }
constexpr size_t kSweepMeta = 16384;  // tot2 (2 × kDigits u32) and the two tickets

size_t fcm_dist_workspace(uint64_t n) {
  if (LCF_ONESWEEP) return 2 * round16(8 * n) + kSweepMeta + 2 * round16(4 * n_sweep_tiles_of(n) * kDigits) + 256;
  return 2 * round16(8 * n) + round16(4 * n_tiles_of(n) * kDigits) + 4 * kDigits + 256;
}

size_t fcm_carry_bytes() { return carry_bytes(); }

// An empty carry (no earlier shard): every per-hash count is 0; the index and
// value areas are never read for a count of 0.
bool fcm_empty_carry(void* carry, cudaStream_t st) { return cudaMemsetAsync(carry, 0, kHashes, st) == cudaSuccess; }

// The FCM distances of x[0, n) (sharded: a shard whose words x[−halo, 0)
// precede it and whose first word has global index gbase; carry = the merged
// summaries of the earlier shards, or null). summary (optional) receives this
// shard's own summary; with match false only the summary is made.
int launch_fcm_shard(const uint64_t* x, uint64_t n, uint32_t halo, uint64_t gbase, const void* carry, void* summary,
                     bool match, void* ws, size_t ws_bytes, cudaStream_t st, uint32_t** dist_out, bool sorted,
                     const uint64_t** sorted_out) {
  (void)ws_bytes;
  uint8_t* p = static_cast<uint8_t*>(ws);
  uint64_t* rec_a = reinterpret_cast<uint64_t*>(p);
  uint64_t* rec_b = reinterpret_cast<uint64_t*>(p + round16(8 * n));
  const uint64_t T = n_tiles_of(n);
  uint32_t* counts = reinterpret_cast<uint32_t*>(p + 2 * round16(8 * n));
  uint32_t* tot = reinterpret_cast<uint32_t*>(p + 2 * round16(8 * n) + round16(4 * T * kDigits));
  uint32_t* dist = reinterpret_cast<uint32_t*>(rec_a);  // pass-1 records are dead after pass 2
  *dist_out = dist;
  if (sorted_out) *sorted_out = rec_b;
  if (n == 0) {
    if (summary) cudaMemsetAsync(summary, 0, kHashes, st);  // no entries
    return 0;
  }
  static const bool init = [] {
    cudaFuncSetAttribute(sort_scatter_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(ScatterSmem));
    cudaFuncSetAttribute(sort_scatter_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(ScatterSmem));
    return true;
  }();
  (void)init;
  int launches = sorted ? 0 : (LCF_ONESWEEP ? 3 : 6);
  if (!sorted && LCF_ONESWEEP) {  // (sorted: rec_b still holds this shard's sorted records from the summary call)
    static const bool init1 = [] {
      cudaFuncSetAttribute(sort_onesweep_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           (int)sizeof(OnesweepSmem));
      cudaFuncSetAttribute(sort_onesweep_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           (int)sizeof(OnesweepSmem));
      return true;
    }();
    (void)init1;
    const uint64_t T1 = n_sweep_tiles_of(n);
    uint8_t* meta = p + 2 * round16(8 * n);
    uint32_t* tot2 = reinterpret_cast<uint32_t*>(meta);
    uint32_t* tick = tot2 + 2 * kDigits;
    uint32_t* st0 = reinterpret_cast<uint32_t*>(meta + kSweepMeta);
    uint32_t* st1 = reinterpret_cast<uint32_t*>(meta + kSweepMeta + round16(4 * T1 * kDigits));
    cudaMemsetAsync(meta, 0, kSweepMeta + 2 * round16(4 * T1 * kDigits), st);
    {
      KTrace kt("fcm_sort_ghist", st);
      const uint64_t ranges = (n + kWarpRecs - 1) / kWarpRecs;
      const unsigned gb = (unsigned)umin64((ranges + kSortWarps - 1) / kSortWarps, 148 * 4);
      sort_ghist_kernel<<<gb, kSortThreads, 0, st>>>(x, n, tot2, halo);
    }
    const int grid = persistent_grid(sort_onesweep_kernel<0>, kST, sizeof(OnesweepSmem), T1);
    {
      KTrace kt("fcm_sort_scatter", st);
      sort_onesweep_kernel<0><<<grid, kST, sizeof(OnesweepSmem), st>>>(x, n, tot2, st0, tick, rec_a, halo);
    }
    {
      KTrace kt("fcm_sort_scatter", st);
      sort_onesweep_kernel<1><<<grid, kST, sizeof(OnesweepSmem), st>>>(rec_a, n, tot2 + kDigits, st1, tick + 1,
                                                                     rec_b, 0);
    }
  } else if (!sorted) {
  {
    KTrace kt("fcm_sort_hist", st);
    sort_hist_kernel<0><<<(unsigned)T, kSortThreads, 0, st>>>(x, n, counts, halo);
  }
  {
    KTrace kt("fcm_sort_scan", st);
    sort_scan_kernel<<<kScanBlocks, kScanWarps * 32, 0, st>>>(counts, (uint32_t)T, tot);
  }
  {
    KTrace kt("fcm_sort_scatter", st);
    sort_scatter_kernel<0><<<(unsigned)T, kST, sizeof(ScatterSmem), st>>>(x, n, counts, tot, rec_a, halo);
  }
  {
    KTrace kt("fcm_sort_hist", st);
    sort_hist_kernel<1><<<(unsigned)T, kSortThreads, 0, st>>>(rec_a, n, counts, 0);
  }
  {
    KTrace kt("fcm_sort_scan", st);
    sort_scan_kernel<<<kScanBlocks, kScanWarps * 32, 0, st>>>(counts, (uint32_t)T, tot);
  }
  {
    KTrace kt("fcm_sort_scatter", st);
    sort_scatter_kernel<1><<<(unsigned)T, kST, sizeof(ScatterSmem), st>>>(rec_a, n, counts, tot, rec_b, 0);
  }
  }
  if (summary) {
    uint8_t* sb = static_cast<uint8_t*>(summary);
    cudaMemsetAsync(sb, 0, kHashes, st);
    KTrace kt("fcm_summary", st);
    fcm_summary_kernel<<<(unsigned)umin64((n + 255) / 256, 148 * 16), 256, 0, st>>>(
        x, n, rec_b, gbase, sb, reinterpret_cast<uint32_t*>(sb + kHashes), reinterpret_cast<uint64_t*>(sb + 17 * kHashes));
    ++launches;
  }
  if (!match) return launches;
  cudaMemsetAsync(dist, 0, 4 * n, st);
  FcmCarry c{nullptr, nullptr, nullptr};
  if (carry) {
    const uint8_t* cb = static_cast<const uint8_t*>(carry);
    c = FcmCarry{cb, reinterpret_cast<const uint32_t*>(cb + kHashes), reinterpret_cast<const uint64_t*>(cb + 17 * kHashes)};
  }
  {
    KTrace kt("fcm_match", st);
    const uint64_t groups = (n + kMatchItems - 1) / kMatchItems;
    const int mblocks = (int)umin64((groups + kMatchBlock - 1) / kMatchBlock, 148 * 16);
    if (carry) {
      fcm_match_kernel<true><<<mblocks, kMatchBlock, 0, st>>>(x, n, rec_b, dist, c, gbase, 0u, 0xFFFFFFFFu);
    } else {
      // LCF_MATCH_SPLIT launches, each writing the distances of one index range
      // only: the scattered writes of a launch then land in an L2-sized part
      // of the distance array
      const uint32_t parts = LCF_MATCH_SPLIT;
      for (uint32_t q = 0; q < parts; ++q) {
        const uint32_t lo = (uint32_t)(n * q / parts), hi = (uint32_t)(n * (q + 1) / parts);
        fcm_match_kernel<false><<<mblocks, kMatchBlock, 0, st>>>(x, n, rec_b, dist, c, gbase, lo, hi);
      }
      launches += parts - 1;
    }
  }
  if (!carry) {  // deferred candidates → distances
    KTrace kt("fcm_verify", st);
    const int vblocks = (int)umin64(((n + 3) / 4 + 255) / 256, 148 * 8);
    fcm_verify_kernel<<<vblocks, 256, 0, st>>>(x, n, rec_b, dist, halo);
    ++launches;
  }
  return launches + 1;
}

int launch_fcm_dist(const uint64_t* x, uint64_t n, void* ws, size_t ws_bytes, cudaStream_t st, uint32_t** dist_out) {
  return launch_fcm_shard(x, n, 0, 0, nullptr, nullptr, true, ws, ws_bytes, st, dist_out, false, nullptr);
}

int launch_fcm_carry_merge(const void* const* summaries, uint32_t count, void* carry, cudaStream_t st) {
  SumPtrs S{};
  for (uint32_t r = 0; r < count && r < 64; ++r) S.p[r] = static_cast<const uint8_t*>(summaries[r]);
  KTrace kt("fcm_carry_merge", st);
  fcm_carry_merge_kernel<<<(unsigned)(kHashes / 256), 256, 0, st>>>(S, count, static_cast<uint8_t*>(carry));
  return 1;
}

}  // namespace lcf
