// lcf_fcm.cuh — the FCM sort record (A-13: hash of x[i−1..i−3], a 12-bit
// fingerprint of x[i], the index) and the one-record match, shared by the
// FCM kernels (lcf_fcm.cu) and the DPratio encoder (lcf_dpratio.cu), which
// verifies the match kernel's deferred candidates.
#pragma once
#include <stdint.h>

namespace lcf {
namespace fcm {

constexpr uint64_t K1 = 0x9E3779B97F4A7C15ull, K2 = 0xC2B2AE3D27D4EB4Full, K3 = 0x165667B19E3779F9ull;
constexpr int kRecHashShift = 44, kRecFpShift = 32;
constexpr uint64_t kRecIdxMask = 0xFFFFFFFFull;
// A deferred candidate in the distance array: distance | kMulti if another
// candidate of the same hash and fingerprint follows in the window.
constexpr uint32_t kMulti = 0x80000000u;

__device__ __forceinline__ uint32_t hi_mul(uint64_t a, uint64_t k) { return (uint32_t)((a * k) >> 32); }

// High hash word of position i of x[0, n); the `halo` words before x[0] are
// its context (a shard's), earlier ones count as 0
__device__ __forceinline__ uint32_t hash_hw(const uint64_t* x, uint64_t i, uint32_t halo) {
  const int64_t j = (int64_t)i;
  const uint64_t a = j - 1 >= -(int64_t)halo ? x[j - 1] : 0, b = j - 2 >= -(int64_t)halo ? x[j - 2] : 0,
                 c = j - 3 >= -(int64_t)halo ? x[j - 3] : 0;
  return hi_mul(a, K1) ^ hi_mul(b, K2) ^ hi_mul(c, K3);
}

// The full match of word i (L174, A-14): its record's sorted position k by
// binary search over rec (sorted by hash, then index), then the nearest of the
// ≤ 4 preceding records of its hash run whose word equals x[i]. The rare
// path: a deferred candidate that failed while others were in the window.
static __device__ __forceinline__ uint32_t match_one(const uint64_t* x, const uint64_t* rec, uint64_t n, uint32_t i,
                                           uint32_t halo) {
  const uint64_t key = ((uint64_t)(hash_hw(x, i, halo) >> 12) << 32) | i;
  uint64_t lo = 0, hi = n;  // first position with key(rec) ≥ key
  while (lo < hi) {
    const uint64_t mid = (lo + hi) / 2;
    const uint64_t r = rec[mid];
    const uint64_t kr = ((r >> kRecHashShift) << 32) | (r & kRecIdxMask);
    if (kr < key) lo = mid + 1;
    else hi = mid;
  }
  if (lo >= n) return 0;
  const uint64_t rk = rec[lo];
  if ((rk & kRecIdxMask) != i) return 0;
  const uint32_t hk = (uint32_t)(rk >> 32);
  const uint64_t xi = x[i];
  for (uint64_t back = 1; back <= 4 && back <= lo; ++back) {
    const uint64_t rb = rec[lo - back];
    const uint32_t hb = (uint32_t)(rb >> 32);
    if ((hb ^ hk) >> 12) break;  // left the hash's run
    const uint32_t jj = (uint32_t)(rb & kRecIdxMask);
    if (hb == hk && x[jj] == xi) return i - jj;
  }
  return 0;
}

}  // namespace fcm
}  // namespace lcf
