// lcf_kernels.cuh — argument blocks and launchers of the codec kernels, plus
// the per-chunk prologue/epilogue shared by all chunk kernels.
#pragma once
#include <map>
#include <mutex>
#include <utility>

#include "lcf_internal.cuh"

namespace lcf {

__host__ __device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }

// Kernel-time tracing (lcf_profile_enable): when enabled, a pair of CUDA
// events brackets every kernel the library launches, on the launching stream.
struct KTrace {
  KTrace(const char* name, cudaStream_t st);
  ~KTrace();
  const char* name;
  cudaStream_t st;
  void* rec;
};

// One compress launch covers chunks [first_chunk, first_chunk + n_chunks) of a
// stream whose input has n_words_total words (FORMAT.md §2).
struct EncArgs {
  const void* in;           // words of chunk first_chunk (16-byte aligned)
  uint64_t n_words_total;   // words of the whole stream input
  uint64_t first_chunk;     // global index of this launch's chunk 0
  uint64_t n_chunks;        // chunks in this launch (grid size)
  uint32_t* table;          // size-table entries of this launch's chunks
  uint8_t* payload;         // where this launch's chunk 0 payload goes
  uint64_t* count_out;      // optional: device u64 ← payload bytes of the launch
  StreamHeader* header;     // optional: full-stream mode writes the header
  uint64_t stream_chunks;   // header n_chunks
  uint64_t n_bytes;         // header n_bytes
  uint64_t payload_total;   // header payload_bytes (lcf_write_header only)
  uint32_t algo, word_bytes;
  uint8_t* pad_start;       // optional zero pad between table and payload base
  uint32_t pad_len;
  // DPratio: FCM side inputs (per-word distance, 0 = no match)
  const uint32_t* fcm_dist;
  // optional pipeline trace (scripts/micro/trace_pipeline.cu): 8 globaltimer
  // stamps per chunk; nullptr in the library
  unsigned long long* trace;
};

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Stamps are compiled in only with -DLCF_TRACE=1 (scripts/build_variants.sh):
// the per-stamp test of a.trace cost ~2 % of the speed encoder's instructions.
#ifndef LCF_TRACE
#define LCF_TRACE 0
#endif
template <class Args>
__device__ __forceinline__ void trace_stamp(const Args& a, uint64_t chunk, int k) {
  if (LCF_TRACE && a.trace) a.trace[chunk * 8 + k] = gtimer();
}

struct DecArgs {
  const uint8_t* stream;  // 16-byte aligned
  uint64_t stream_bytes;
  uint8_t* out;           // 16-byte aligned
  uint64_t out_capacity;
  uint32_t algo, word_bytes;
  uint32_t* tile_flag;    // DPratio: per-tile completion (epoch) flags
  unsigned long long* trace;  // lcf__trace_decompress only: 8 globaltimer stamps per chunk / tile
  // DPratio tile-range decode (pipelined host path): tiles [first_tile,
  // end_tile) only (end_tile 0: all); base_off = payload offset of chunk
  // 2·first_tile; earlier tiles are already final in `out` (an earlier launch
  // on the same stream) and only their payload bytes may be absent.
  uint64_t first_tile, end_tile, base_off;
  // DPratio: word 0 of this stream is global word gbase (0, or a shard's first
  // word, NEXT-1). A word whose distance reaches before it, or into a tile not
  // yet complete, is left pending: the output holds the global index it
  // copies and its bit in `pend` (1 bit per word; every decoded tile writes
  // its bitmap words) is set; any_pend ← epoch if any word is.
  uint64_t gbase;
  uint32_t* pend;
  uint32_t* tgt;       // bitmap of the words some pending word points at (chain nodes)
  uint32_t* any_pend;
  // (optional) list of the chain nodes, appended as they are first marked,
  // and its length (zeroed before the launch)
  uint32_t* nodes;
  uint32_t* n_nodes;
};

// The pending-word views of the DPratio root resolution (dp_find_roots /
// dp_gather_roots in lcf_dpratio.cu): view q covers global words
// [first, first + n) at `out` with bitmap `pend` (device pointers, local or
// CUDA-IPC-mapped peers), sorted by first and contiguous.
constexpr uint32_t kMaxViews = 64;
struct DpView {
  uint64_t first, n;
  uint64_t* out;
  uint32_t* pend;
  uint32_t* tgt;  // chain-node marks (same indexing as pend)
};
struct DpViews {
  uint32_t count, self;
  DpView v[kMaxViews];
};

struct DecChunk {
  uint64_t c;              // chunk index (DPratio: tile index)
  uint64_t base;           // payload base offset in the stream
  uint64_t payload_bytes;
  uint64_t n_words;        // words of the whole output
  uint64_t n_chunks;
  uint32_t len, m, raw, ok;
};

__device__ __forceinline__ void finish_encode(const EncArgs& a, uint64_t total) {
  if (a.count_out) *a.count_out = total;
  if (a.header) {
    uint32_t w[8];
    w[0] = kMagic;
    w[1] = kVersion | (a.algo << 8) | (a.word_bytes << 16);
    w[2] = (uint32_t)a.n_bytes; w[3] = (uint32_t)(a.n_bytes >> 32);
    w[4] = (uint32_t)a.stream_chunks; w[5] = (uint32_t)(a.stream_chunks >> 32);
    w[6] = (uint32_t)total; w[7] = (uint32_t)(total >> 32);
    uint4* h = reinterpret_cast<uint4*>(a.header);
    h[0] = make_uint4(w[0], w[1], w[2], w[3]);
    h[1] = make_uint4(w[4], w[5], w[6], w[7]);
  }
}

// Reads and validates the stream header (FORMAT.md §1, §7). Returns false for
// a malformed header; fills n_words/n_chunks/base/payload_bytes.
__device__ __forceinline__ bool read_header(const DecArgs& a, const LaunchCtx& ctx, uint64_t& n_words,
                                            uint64_t& n_chunks, uint64_t& base, uint64_t& payload) {
  if (a.stream_bytes < kHeaderBytes) return false;
  const uint4 h0 = reinterpret_cast<const uint4*>(a.stream)[0];
  const uint4 h1 = reinterpret_cast<const uint4*>(a.stream)[1];
  const uint64_t n_bytes = ((uint64_t)h0.w << 32) | h0.z;
  n_chunks = ((uint64_t)h1.y << 32) | h1.x;
  payload = ((uint64_t)h1.w << 32) | h1.z;
  if (h0.x != kMagic || (h0.y & 0xFF) != kVersion || ((h0.y >> 8) & 0xFF) != a.algo ||
      ((h0.y >> 16) & 0xFF) != a.word_bytes || (h0.y >> 24) != 0)
    return false;
  if (n_bytes % a.word_bytes) return false;
  n_words = n_bytes / a.word_bytes;
  const uint64_t expect = a.algo == DPRATIO ? 2 * ((n_words + 2047) / 2048)
                                            : (n_bytes + kChunkBytes - 1) / kChunkBytes;
  if (n_chunks != expect) return false;
  base = round16(kHeaderBytes + 4 * n_chunks);
  if (base > a.stream_bytes || payload > a.stream_bytes - base) return false;
  return true;
}

// Grid of a persistent kernel: every SM filled to its occupancy, capped by the
// amount of work. The resident capacity is computed once per (kernel, device):
// the occupancy query costs microseconds of host time that would otherwise sit
// between the caller's start event and the launch.
inline int resident_capacity(const void* kernel, int threads, size_t smem) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, int> cache;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> g(mu);
  auto key = std::make_pair(kernel, dev);
  auto it = cache.find(key);
  if (it != cache.end()) return it->second;
  int sms = 0, per_sm = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, threads, smem);
  if (per_sm < 1) per_sm = 1;
  return cache[key] = sms * per_sm;
}
template <typename Kern> int persistent_grid(Kern kernel, int threads, size_t smem, uint64_t work) {
  const uint64_t g = (uint64_t)resident_capacity(reinterpret_cast<const void*>(kernel), threads, smem);
  return (int)(work < g ? (work ? work : 1) : g);
}

template <typename U> void launch_speed_encode(const EncArgs& a, const LaunchCtx& ctx, cudaStream_t st);
template <typename U>
void launch_speed_decode(const DecArgs& a, const LaunchCtx& ctx, uint64_t max_chunks, cudaStream_t st);
void launch_spratio_encode(const EncArgs& a, const LaunchCtx& ctx, cudaStream_t st);
void launch_spratio_decode(const DecArgs& a, const LaunchCtx& ctx, uint64_t max_chunks, cudaStream_t st);
void launch_write_header(const EncArgs& a, cudaStream_t st);
// FCM distances of n words at x (lcf_fcm.cu): workspace bytes, and the launch
// (returns the number of kernels; *dist points into ws, n u32 values).
size_t fcm_dist_workspace(uint64_t n_words);
int launch_fcm_dist(const uint64_t* x, uint64_t n, void* ws, size_t ws_bytes, cudaStream_t st, uint32_t** dist);
// Sharded DPratio (NEXT-1, lcf_fcm.cu): the same over a shard with `halo`
// context words before x, global first index gbase, the merged summaries of
// earlier shards (carry, nullable); `summary` (nullable) receives this
// shard's summary (fcm_carry_bytes() bytes); match = false: summary only.
size_t fcm_carry_bytes();
bool fcm_empty_carry(void* carry, cudaStream_t st);
int launch_fcm_shard(const uint64_t* x, uint64_t n, uint32_t halo, uint64_t gbase, const void* carry, void* summary,
                     bool match, void* ws, size_t ws_bytes, cudaStream_t st, uint32_t** dist, bool sorted = false,
                     const uint64_t** sorted_out = nullptr);
// summaries: host array of `count` (≤ 64) device pointers, shard order
int launch_fcm_carry_merge(const void* const* summaries, uint32_t count, void* carry, cudaStream_t st);
size_t dpratio_fcm_workspace(uint64_t n_words);
int launch_dpratio_encode(const EncArgs& a, const LaunchCtx& ctx, void* ws, size_t ws_bytes, cudaStream_t st,
                          uint32_t halo = 0, uint64_t gbase = 0, const void* carry = nullptr, bool sorted = false);
void launch_dpratio_decode(const DecArgs& a, const LaunchCtx& ctx, uint64_t max_tiles, cudaStream_t st);
// Root resolution of pending words of view `self`, local words [w_lo, w_hi)
// (clamped to the stream header's word count when `stream` is given).
// find: every pending word's target becomes its chain's root (a final word),
// with path compression — mode 0 walks the marked chain nodes only, mode 1
// the other pending words (whose walks then end after a hop or two), mode 2
// all of them; gather: pending words take their root's value and both
// bitmaps are cleared (mode 2; single view: mode 0 the leaves through their
// chain nodes — no leaf walk needed — then mode 1 the chain nodes). Every view's decode must be complete before any
// find, and every find before any gather. any_pend (nullable): skip unless
// *any_pend == ctx.epoch.
void launch_dp_find_roots(const DpViews& v, const uint8_t* stream, uint64_t w_lo, uint64_t w_hi,
                          const LaunchCtx& ctx, const uint32_t* any_pend, cudaStream_t st, int mode = 2);
void launch_dp_gather_roots(const DpViews& v, const uint8_t* stream, uint64_t w_lo, uint64_t w_hi,
                            const LaunchCtx& ctx, const uint32_t* any_pend, cudaStream_t st, int mode = 2);
// Single view with the decoder's chain-node list (nodes[0, *n_nodes), local
// indices): walk the chain nodes to their roots (gather = false), or give them
// their roots' values (gather = true; after the leaves' gather). `cap` bounds
// the list (max_words).
void launch_dp_gather_leaves(const DpView& v, const uint8_t* stream, uint64_t w_lo, uint64_t w_hi,
                             const LaunchCtx& ctx, const uint32_t* any_pend, cudaStream_t st);
void launch_dp_nodes(const DpView& v, const uint32_t* nodes, const uint32_t* n_nodes, uint64_t cap,
                     const LaunchCtx& ctx, const uint32_t* any_pend, bool gather, cudaStream_t st);

}  // namespace lcf
