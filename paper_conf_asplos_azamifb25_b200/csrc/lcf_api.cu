// lcf_api.cu — host side of liblcf.so: the C ABI of include/lcf.h, argument
// validation, per-(device, stream) workspaces, launch of the codec kernels.
#include <lcf.h>

#include <atomic>
#include <cstdlib>
#include <cstring>
#include <map>
#include <string>
#include <mutex>
#include <utility>
#include <vector>

#include "lcf_kernels.cuh"

using namespace lcf;

namespace {

std::atomic<uint64_t> g_launches{0};
unsigned long long* g_trace_buf = nullptr;  // lcf__trace_compress only
unsigned long long* g_trace_dec = nullptr;  // lcf__trace_decompress only

struct Workspace {
  int device = -1;
  cudaStream_t stream = nullptr;
  std::mutex mu;
  unsigned long long* ticket = nullptr;  // [0] ticket counter, [1] retired CTAs (kernels reset both)
  uint64_t* status = nullptr;            // look-back status words
  size_t status_cap = 0;
  uint32_t* tile_flag = nullptr;         // DPratio decode tile completion flags
  size_t tile_cap = 0;
  uint32_t* pend = nullptr;              // DPratio decode pending-word bitmap (1 bit per word)
  size_t pend_cap = 0;
  uint32_t* tgt = nullptr;               // DPratio decode chain-node marks (1 bit per word)
  size_t tgt_cap = 0;
  uint32_t* nodes = nullptr;             // DPratio decode chain-node list: [0] count, then indices
  size_t nodes_cap = 0;
  uint32_t* any_pend = nullptr;          // DPratio decode: epoch of the newest launch with a pending word
  uint32_t* err = nullptr;               // (epoch << 8 | bits) of the newest failure
  uint32_t epoch = 0, checked_epoch = 0;
  void* scratch[4] = {nullptr, nullptr, nullptr, nullptr};  // grown on demand
  size_t scratch_cap[4] = {0, 0, 0, 0};
  // pipelined host path: copy streams, per-slice events, pinned staging
  std::mutex host_mu;
  cudaStream_t h2d = nullptr, d2h = nullptr;
  std::vector<cudaEvent_t> ev;
  uint8_t* hstage = nullptr;
  size_t hstage_cap = 0;
  // sharded DPratio: scratch[2] holds the sorted FCM records of this shard
  // (set by lcf_dpratio_shard_summary, consumed by the next compress_shard)
  const void* sorted_x = nullptr;
  const void* sorted_ws = nullptr;
  uint64_t sorted_n = 0, sorted_first = 0;
};

std::mutex g_mu;
std::map<std::pair<int, cudaStream_t>, Workspace*> g_ws;

constexpr uint32_t kEpochLimit = 1u << 22;

bool cuda_ok(cudaError_t e) { return e == cudaSuccess; }

Workspace* get_ws(cudaStream_t stream, lcf_status_t* st) {
  int dev = -1;
  if (!cuda_ok(cudaGetDevice(&dev))) { *st = LCF_ERROR_CUDA; return nullptr; }
  std::lock_guard<std::mutex> g(g_mu);
  auto key = std::make_pair(dev, stream);
  auto it = g_ws.find(key);
  if (it != g_ws.end()) return it->second;
  Workspace* ws = new Workspace();
  ws->device = dev;
  ws->stream = stream;
  if (!cuda_ok(cudaMalloc(&ws->ticket, 2 * sizeof(unsigned long long))) ||
      !cuda_ok(cudaMalloc(&ws->err, sizeof(uint32_t))) || !cuda_ok(cudaMalloc(&ws->any_pend, sizeof(uint32_t))) ||
      !cuda_ok(cudaMemsetAsync(ws->any_pend, 0, sizeof(uint32_t), stream)) ||
      !cuda_ok(cudaMemsetAsync(ws->ticket, 0, 2 * sizeof(unsigned long long), stream)) ||
      !cuda_ok(cudaMemsetAsync(ws->err, 0, sizeof(uint32_t), stream))) {
    *st = LCF_ERROR_OUT_OF_MEMORY;
    delete ws;
    return nullptr;
  }
  g_ws[key] = ws;
  return ws;
}

template <typename T>
lcf_status_t grow(T*& ptr, size_t& cap, size_t need, cudaStream_t s, bool zero) {
  if (cap >= need) return LCF_SUCCESS;
  size_t ncap = cap * 2 > need ? cap * 2 : need;
  if (ptr) {
    cudaStreamSynchronize(s);
    cudaFree(ptr);
    ptr = nullptr;
    cap = 0;
  }
  if (!cuda_ok(cudaMalloc(&ptr, ncap * sizeof(T)))) return LCF_ERROR_OUT_OF_MEMORY;
  if (zero && !cuda_ok(cudaMemsetAsync(ptr, 0, ncap * sizeof(T), s))) return LCF_ERROR_CUDA;
  cap = ncap;
  return LCF_SUCCESS;
}

uint32_t next_epoch(Workspace* ws) {
  if (++ws->epoch >= kEpochLimit) {  // wrap: forget every status/flag word
    if (ws->status) cudaMemsetAsync(ws->status, 0, ws->status_cap * sizeof(uint64_t), ws->stream);
    if (ws->tile_flag) cudaMemsetAsync(ws->tile_flag, 0, ws->tile_cap * sizeof(uint32_t), ws->stream);
    if (ws->any_pend) cudaMemsetAsync(ws->any_pend, 0, sizeof(uint32_t), ws->stream);
    cudaMemsetAsync(ws->err, 0, sizeof(uint32_t), ws->stream);
    ws->epoch = 1;
    ws->checked_epoch = 0;
  }
  return ws->epoch;
}

LaunchCtx make_ctx(Workspace* ws) {
  LaunchCtx c;
  c.ticket = ws->ticket;
  c.status = ws->status;
  c.epoch = next_epoch(ws);
  c.err = ws->err;
  return c;
}

uint32_t word_bytes_of(int algo) { return (algo == LCF_SPSPEED || algo == LCF_SPRATIO) ? 4u : 8u; }
bool valid_algo(int algo) { return algo >= LCF_SPSPEED && algo <= LCF_DPRATIO; }
bool dtype_matches(int algo, int dtype) {
  return (word_bytes_of(algo) == 4 && dtype == LCF_FLOAT32) || (word_bytes_of(algo) == 8 && dtype == LCF_FLOAT64);
}
bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

uint64_t payload_bound(int algo, uint64_t in_bytes) {
  const uint64_t wb = word_bytes_of(algo);
  if (algo == LCF_DPRATIO) {
    const uint64_t n = in_bytes / wb;
    return 2 * ((n / 2048) * 16384 + round16(8 * (n % 2048)));
  }
  return (in_bytes / kChunkBytes) * kChunkBytes + round16(in_bytes % kChunkBytes);
}

// Host-side header check (same rules as lcf::read_header).
lcf_status_t check_header(const uint8_t* h, uint64_t in_bytes, int algo, uint64_t* n_bytes, uint64_t* n_chunks,
                          uint64_t* payload) {
  uint32_t magic;
  std::memcpy(&magic, h, 4);
  if (magic != kMagic || h[4] != kVersion || h[7] != 0 || h[5] > 3) return LCF_ERROR_CORRUPT_STREAM;
  if (h[5] != algo) return LCF_ERROR_DTYPE_MISMATCH;
  if (h[6] != word_bytes_of(algo)) return LCF_ERROR_CORRUPT_STREAM;
  std::memcpy(n_bytes, h + 8, 8);
  std::memcpy(n_chunks, h + 16, 8);
  std::memcpy(payload, h + 24, 8);
  if (*n_bytes % h[6]) return LCF_ERROR_CORRUPT_STREAM;
  if (*n_chunks != lcf_num_chunks((lcf_algo_t)algo, *n_bytes)) return LCF_ERROR_CORRUPT_STREAM;
  if (*n_chunks > (in_bytes - 32) / 4) return LCF_ERROR_CORRUPT_STREAM;
  const uint64_t base = round16(kHeaderBytes + 4 * *n_chunks);
  if (base > in_bytes || *payload > in_bytes - base) return LCF_ERROR_CORRUPT_STREAM;
  return LCF_SUCCESS;
}

lcf_status_t last_launch_status() {
  return cuda_ok(cudaGetLastError()) ? LCF_SUCCESS : LCF_ERROR_CUDA;
}

lcf_status_t device_error_since(Workspace* ws, uint32_t since_epoch) {
  uint32_t e = 0;
  if (!cuda_ok(cudaMemcpyAsync(&e, ws->err, 4, cudaMemcpyDeviceToHost, ws->stream)) ||
      !cuda_ok(cudaStreamSynchronize(ws->stream)))
    return LCF_ERROR_CUDA;
  if ((e >> 8) > since_epoch) return (e & DERR_SMALL) ? LCF_ERROR_BUFFER_TOO_SMALL : LCF_ERROR_CORRUPT_STREAM;
  return LCF_SUCCESS;
}

EncArgs enc_args(int algo, const void* in, uint64_t in_bytes) {
  EncArgs a{};
  a.in = in;
  a.word_bytes = word_bytes_of(algo);
  a.n_words_total = in_bytes / a.word_bytes;
  a.algo = (uint32_t)algo;
  a.n_bytes = in_bytes;
  return a;
}

lcf_status_t enqueue_encode(Workspace* ws, EncArgs& a) {
  if (lcf_status_t s = grow(ws->status, ws->status_cap, a.n_chunks, ws->stream, true)) return s;
  if (a.algo == LCF_DPRATIO) {
    ws->sorted_x = nullptr;  // scratch[2] is rewritten
    const size_t need = dpratio_fcm_workspace(a.n_words_total);
    if (lcf_status_t s = grow(reinterpret_cast<uint8_t*&>(ws->scratch[2]), ws->scratch_cap[2], need, ws->stream, false))
      return s;
    LaunchCtx ctx = make_ctx(ws);
    g_launches += launch_dpratio_encode(a, ctx, ws->scratch[2], ws->scratch_cap[2], ws->stream);
    return last_launch_status();
  }
  LaunchCtx ctx = make_ctx(ws);
  switch (a.algo) {
    case LCF_SPSPEED: launch_speed_encode<uint32_t>(a, ctx, ws->stream); break;
    case LCF_DPSPEED: launch_speed_encode<uint64_t>(a, ctx, ws->stream); break;
    case LCF_SPRATIO: launch_spratio_encode(a, ctx, ws->stream); break;
    default: return LCF_ERROR_INVALID_ARGUMENT;
  }
  ++g_launches;
  return last_launch_status();
}

}  // namespace

extern "C" {

uint64_t lcf_num_chunks(lcf_algo_t algo, size_t in_bytes) {
  if (!valid_algo(algo)) return 0;
  const uint64_t wb = word_bytes_of(algo);
  if (algo == LCF_DPRATIO) return 2 * ((in_bytes / wb + 2047) / 2048);
  return (in_bytes + kChunkBytes - 1) / kChunkBytes;
}

size_t lcf_max_compressed_size(lcf_algo_t algo, lcf_dtype_t dtype, size_t in_bytes) {
  (void)dtype;
  if (!valid_algo(algo)) return 0;
  return round16(kHeaderBytes + 4 * lcf_num_chunks(algo, in_bytes)) + payload_bound(algo, in_bytes);
}

uint64_t lcf_launch_count(void) { return g_launches.load(); }

// Undocumented diagnostic entry point (not in lcf.h): lcf_compress that also
// records 8 globaltimer stamps per chunk into d_trace (n_chunks × 8 u64) for the
// speed codecs' pipeline analysis (scripts/trace_pipeline.py).
lcf_status_t lcf__trace_compress(lcf_algo_t algo, lcf_dtype_t dtype, const void* d_in, size_t in_bytes, void* d_out,
                                 size_t out_capacity, unsigned long long* d_trace, void* stream) {
  g_trace_buf = d_trace;
  size_t n = 0;
  lcf_status_t st = lcf_compress(algo, dtype, d_in, in_bytes, d_out, out_capacity, &n, stream);
  g_trace_buf = nullptr;
  return st;
}

// Diagnostic twin of lcf_decompress (not in lcf.h): DPratio decode kernels
// record 8 globaltimer stamps per tile into d_trace (n_tiles × 8 u64).
lcf_status_t lcf__trace_decompress(lcf_algo_t algo, lcf_dtype_t dtype, const void* d_in, size_t in_bytes,
                                   void* d_out, size_t out_capacity, unsigned long long* d_trace, void* stream) {
  g_trace_dec = d_trace;
  size_t n = 0;
  lcf_status_t st = lcf_decompress(algo, dtype, d_in, in_bytes, d_out, out_capacity, &n, stream);
  g_trace_dec = nullptr;
  return st;
}

lcf_status_t lcf_compress(lcf_algo_t algo, lcf_dtype_t dtype, const void* d_in, size_t in_bytes, void* d_out,
                          size_t out_capacity, size_t* out_bytes, void* stream_) {
  cudaStream_t stream = (cudaStream_t)stream_;
  if (!valid_algo(algo)) return LCF_ERROR_INVALID_ARGUMENT;
  if (!dtype_matches(algo, dtype)) return LCF_ERROR_DTYPE_MISMATCH;
  const uint32_t wb = word_bytes_of(algo);
  if (in_bytes % wb || !d_out || !aligned16(d_out) || (in_bytes && (!d_in || !aligned16(d_in))))
    return LCF_ERROR_INVALID_ARGUMENT;
  if (out_capacity < lcf_max_compressed_size(algo, dtype, in_bytes)) return LCF_ERROR_BUFFER_TOO_SMALL;
  if (algo == LCF_DPRATIO && in_bytes / 8 >= (1ull << 31)) return LCF_ERROR_INVALID_ARGUMENT;  // 32-bit FCM record index
  lcf_status_t st = LCF_SUCCESS;
  Workspace* ws = get_ws(stream, &st);
  if (!ws) return st;
  std::lock_guard<std::mutex> g(ws->mu);
  const uint64_t C = lcf_num_chunks(algo, in_bytes);
  const uint64_t base = round16(kHeaderBytes + 4 * C);
  EncArgs a = enc_args(algo, d_in, in_bytes);
  a.first_chunk = 0;
  a.n_chunks = C;
  a.stream_chunks = C;
  a.table = reinterpret_cast<uint32_t*>(static_cast<uint8_t*>(d_out) + kHeaderBytes);
  a.payload = static_cast<uint8_t*>(d_out) + base;
  a.header = reinterpret_cast<StreamHeader*>(d_out);
  a.pad_start = static_cast<uint8_t*>(d_out) + kHeaderBytes + 4 * C;
  a.pad_len = (uint32_t)(base - kHeaderBytes - 4 * C);
  a.trace = g_trace_buf;
  if (C == 0) {
    launch_write_header(a, stream);
    ++g_launches;
    st = last_launch_status();
  } else {
    st = enqueue_encode(ws, a);
  }
  if (st) return st;
  if (out_bytes) {
    uint64_t pb = 0;
    if (!cuda_ok(cudaMemcpyAsync(&pb, static_cast<uint8_t*>(d_out) + 24, 8, cudaMemcpyDeviceToHost, stream)) ||
        !cuda_ok(cudaStreamSynchronize(stream)))
      return LCF_ERROR_CUDA;
    *out_bytes = base + pb;
  }
  return LCF_SUCCESS;
}

// The DPratio decode of tiles [first_tile, end_tile) (end 0: all) of the stream
// at a.stream into a.out: the tile decoder, then the root resolution of the
// words it left pending (single view: the whole output). Caller holds ws->mu.
static lcf_status_t dpratio_decode_range(Workspace* ws, DecArgs a, const LaunchCtx& ctx, uint64_t max_tiles,
                                         uint64_t end_tile, cudaStream_t stream) {
  const uint64_t words = a.out_capacity / 8, W = (words + 31) / 32 + 1;
  lcf_status_t st;
  // (each bitmap in its own buffer: the layout must not depend on the call's
  // size, since every call leaves both bitmaps zero only where it wrote)
  if ((st = grow(ws->pend, ws->pend_cap, W, stream, true)) || (st = grow(ws->tgt, ws->tgt_cap, W, stream, true)) ||
      (st = grow(ws->nodes, ws->nodes_cap, words + 4, stream, false)))
    return st;
  uint32_t* cnt = ws->nodes;
  a.pend = ws->pend;
  a.tgt = ws->tgt;
  a.any_pend = ws->any_pend;
  a.n_nodes = cnt;
  a.nodes = cnt + 4;
  if (!cuda_ok(cudaMemsetAsync(cnt, 0, 4, stream))) return LCF_ERROR_CUDA;
  launch_dpratio_decode(a, ctx, max_tiles, stream);
  DpViews v{};
  v.count = 1;
  v.self = 0;
  v.v[0] = DpView{0, words, reinterpret_cast<uint64_t*>(a.out), ws->pend, ws->tgt};
  const uint64_t lo = a.first_tile * 2048, hi = end_tile && end_tile * 2048 < words ? end_tile * 2048 : words;
  launch_dp_nodes(v.v[0], a.nodes, cnt, words, ctx, ws->any_pend, false, stream);  // chain nodes → roots
  launch_dp_gather_leaves(v.v[0], a.stream, lo, hi, ctx, ws->any_pend, stream);    // leaves, via their chain node
  launch_dp_nodes(v.v[0], a.nodes, cnt, words, ctx, ws->any_pend, true, stream);   // chain nodes
  g_launches += 3;
  // both bitmaps of the range back to zero (the next launch writes its tiles' words)
  if (hi > lo && (!cuda_ok(cudaMemsetAsync(ws->pend + lo / 32, 0, 4 * ((hi + 31) / 32 - lo / 32), stream)) ||
                  !cuda_ok(cudaMemsetAsync(ws->tgt + lo / 32, 0, 4 * ((hi + 31) / 32 - lo / 32), stream))))
    return LCF_ERROR_CUDA;
  return LCF_SUCCESS;
}

lcf_status_t lcf_decompress(lcf_algo_t algo, lcf_dtype_t dtype, const void* d_in, size_t in_bytes, void* d_out,
                            size_t out_capacity, size_t* out_bytes, void* stream_) {
  cudaStream_t stream = (cudaStream_t)stream_;
  if (!valid_algo(algo)) return LCF_ERROR_INVALID_ARGUMENT;
  if (!dtype_matches(algo, dtype)) return LCF_ERROR_DTYPE_MISMATCH;
  if (!d_in || !aligned16(d_in) || (out_capacity && (!d_out || !aligned16(d_out))))
    return LCF_ERROR_INVALID_ARGUMENT;
  if (in_bytes < kHeaderBytes) return LCF_ERROR_CORRUPT_STREAM;
  lcf_status_t st = LCF_SUCCESS;
  Workspace* ws = get_ws(stream, &st);
  if (!ws) return st;
  std::lock_guard<std::mutex> g(ws->mu);
  uint64_t grid;
  uint64_t n_bytes = 0;
  if (out_bytes) {
    uint8_t h[32];
    if (!cuda_ok(cudaMemcpyAsync(h, d_in, 32, cudaMemcpyDeviceToHost, stream)) ||
        !cuda_ok(cudaStreamSynchronize(stream)))
      return LCF_ERROR_CUDA;
    uint64_t n_chunks, payload;
    if (lcf_status_t s = check_header(h, in_bytes, algo, &n_bytes, &n_chunks, &payload)) return s;
    if (n_bytes > out_capacity) return LCF_ERROR_BUFFER_TOO_SMALL;
    grid = n_chunks;
    if (grid == 0) {
      *out_bytes = 0;
      return LCF_SUCCESS;
    }
  } else {
    const uint64_t by_table = (in_bytes - kHeaderBytes) / 4;
    const uint64_t by_out = (algo == LCF_DPRATIO ? 2 : 1) * ((out_capacity + kChunkBytes - 1) / kChunkBytes);
    grid = by_table < by_out ? by_table : by_out;
    if (grid == 0) grid = 1;  // still validate the header on the device
  }
  if (lcf_status_t s = grow(ws->status, ws->status_cap, grid, stream, true)) return s;
  if (algo == LCF_DPRATIO)
    if (lcf_status_t s = grow(ws->tile_flag, ws->tile_cap, grid / 2 + 1, stream, true)) return s;
  DecArgs a{};
  a.trace = g_trace_dec;
  a.stream = static_cast<const uint8_t*>(d_in);
  a.stream_bytes = in_bytes;
  a.out = static_cast<uint8_t*>(d_out);
  a.out_capacity = out_capacity;
  a.algo = (uint32_t)algo;
  a.word_bytes = word_bytes_of(algo);
  a.tile_flag = ws->tile_flag;
  LaunchCtx ctx = make_ctx(ws);
  switch (algo) {
    case LCF_SPSPEED: launch_speed_decode<uint32_t>(a, ctx, grid, stream); break;
    case LCF_DPSPEED: launch_speed_decode<uint64_t>(a, ctx, grid, stream); break;
    case LCF_SPRATIO: launch_spratio_decode(a, ctx, grid, stream); break;
    case LCF_DPRATIO:
      if ((st = dpratio_decode_range(ws, a, ctx, grid / 2 + 1, 0, stream))) return st;
      break;
    default: return LCF_ERROR_INVALID_ARGUMENT;
  }
  ++g_launches;
  if ((st = last_launch_status())) return st;
  if (out_bytes) {
    // a synchronising call reports any device-found failure since the last
    // report on this stream (include/lcf.h), its own included
    st = device_error_since(ws, ws->checked_epoch);
    ws->checked_epoch = ws->epoch;
    if (st) return st;
    *out_bytes = n_bytes;
  }
  return LCF_SUCCESS;
}

lcf_status_t lcf_get_info(const void* d_in, size_t in_bytes, lcf_algo_t* algo, lcf_dtype_t* dtype,
                          size_t* uncompressed_bytes, size_t* compressed_bytes, void* stream_) {
  cudaStream_t stream = (cudaStream_t)stream_;
  if (!d_in) return LCF_ERROR_INVALID_ARGUMENT;
  if (in_bytes < kHeaderBytes) return LCF_ERROR_CORRUPT_STREAM;
  uint8_t h[32];
  if (!cuda_ok(cudaMemcpyAsync(h, d_in, 32, cudaMemcpyDeviceToHost, stream)) ||
      !cuda_ok(cudaStreamSynchronize(stream)))
    return LCF_ERROR_CUDA;
  if (h[5] > 3) return LCF_ERROR_CORRUPT_STREAM;
  uint64_t nb, nc, pb;
  if (lcf_status_t s = check_header(h, in_bytes, h[5], &nb, &nc, &pb)) return s;
  if (algo) *algo = (lcf_algo_t)h[5];
  if (dtype) *dtype = h[6] == 4 ? LCF_FLOAT32 : LCF_FLOAT64;
  if (uncompressed_bytes) *uncompressed_bytes = nb;
  if (compressed_bytes) *compressed_bytes = round16(kHeaderBytes + 4 * nc) + pb;
  return LCF_SUCCESS;
}

lcf_status_t lcf_check_stream(void* stream_) {
  cudaStream_t stream = (cudaStream_t)stream_;
  lcf_status_t st = LCF_SUCCESS;
  Workspace* ws = get_ws(stream, &st);
  if (!ws) return st;
  std::lock_guard<std::mutex> g(ws->mu);
  st = device_error_since(ws, ws->checked_epoch);
  ws->checked_epoch = ws->epoch;
  return st;
}

// ---- pipelined host path (chunk-local codecs) -------------------------------
// The input is cut into slices of whole chunks. Chunk encodings are
// context-free (L104), so slice i compressed on its own is an LCF1 sub-stream
// whose table entries and padded payloads are exactly those of chunks
// [c0, c1) of the whole stream; the host stitches header ‖ table slices ‖
// payload slices (FORMAT.md) — the same bytes lcf_compress writes. The H2D of
// slice i+1, the codec on slice i and the D2H of slice i−1 run on three
// streams, so the two PCIe directions overlap each other and the kernels.
// Decompression mirrors it: per slice, a sub-header and table slice built on
// the host go up with the slice's payload bytes; the decoded words come back
// while later slices decode. DPratio is not chunk-local (FCM, L170) and keeps
// the serial path.
static uint64_t host_slice_chunks(uint64_t C) {
  uint64_t want = 0;
  if (const char* e = std::getenv("LCF_HOST_SLICE_BYTES")) want = std::strtoull(e, nullptr, 10) / kChunkBytes;
  if (want == 0) {  // ~8 slices, 4..64 MiB each
    want = (C + 7) / 8;
    const uint64_t lo = (4ull << 20) / kChunkBytes, hi = (64ull << 20) / kChunkBytes;
    want = want < lo ? lo : want > hi ? hi : want;
  }
  return want;
}

static lcf_status_t host_pipe_init(Workspace* ws, size_t n_events, size_t stage_bytes) {
  if (!ws->h2d && (!cuda_ok(cudaStreamCreateWithFlags(&ws->h2d, cudaStreamNonBlocking)) ||
                   !cuda_ok(cudaStreamCreateWithFlags(&ws->d2h, cudaStreamNonBlocking))))
    return LCF_ERROR_CUDA;
  while (ws->ev.size() < n_events) {
    cudaEvent_t e;
    if (!cuda_ok(cudaEventCreateWithFlags(&e, cudaEventDisableTiming))) return LCF_ERROR_CUDA;
    ws->ev.push_back(e);
  }
  if (ws->hstage_cap < stage_bytes) {
    if (ws->hstage) cudaFreeHost(ws->hstage);
    ws->hstage = nullptr;
    ws->hstage_cap = 0;
    if (!cuda_ok(cudaMallocHost(&ws->hstage, stage_bytes))) return LCF_ERROR_OUT_OF_MEMORY;
    ws->hstage_cap = stage_bytes;
  }
  return LCF_SUCCESS;
}

static void put_header(uint8_t* h, int algo, uint64_t n_bytes, uint64_t n_chunks, uint64_t payload) {
  const uint32_t w0 = kMagic, w1 = kVersion | ((uint32_t)algo << 8) | (word_bytes_of(algo) << 16);
  std::memcpy(h, &w0, 4);
  std::memcpy(h + 4, &w1, 4);
  std::memcpy(h + 8, &n_bytes, 8);
  std::memcpy(h + 16, &n_chunks, 8);
  std::memcpy(h + 24, &payload, 8);
}

static lcf_status_t compress_host_pipelined(lcf_algo_t algo, lcf_dtype_t dtype, const uint8_t* h_in, size_t in_bytes,
                                     uint8_t* h_out, size_t out_capacity, size_t* out_bytes, Workspace* ws,
                                     uint64_t C, uint64_t sc) {
  const uint64_t k = (C + sc - 1) / sc;
  const uint64_t base = round16(kHeaderBytes + 4 * C);
  if (out_capacity < base) return LCF_ERROR_BUFFER_TOO_SMALL;
  const size_t sub_cap = lcf_max_compressed_size(algo, dtype, sc * kChunkBytes);
  lcf_status_t st;
  if ((st = host_pipe_init(ws, 2 * k, 32 * k))) return st;
  {
    std::lock_guard<std::mutex> g(ws->mu);
    if ((st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[0]), ws->scratch_cap[0], round16(in_bytes) + 16,
                   ws->stream, false)) ||
        (st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[1]), ws->scratch_cap[1], k * sub_cap, ws->stream, false)))
      return st;
  }
  uint8_t* d_in = static_cast<uint8_t*>(ws->scratch[0]);
  uint8_t* d_sub = static_cast<uint8_t*>(ws->scratch[1]);
  cudaEvent_t* evH = ws->ev.data();
  cudaEvent_t* evC = ws->ev.data() + k;
  uint64_t off = base;  // next payload byte of the stitched stream
  auto finish = [&](uint64_t i) -> lcf_status_t {
    const uint64_t c0 = i * sc, kc = (c0 + sc < C ? sc : C - c0);
    const uint64_t sbase = round16(kHeaderBytes + 4 * kc);
    if (!cuda_ok(cudaEventSynchronize(evC[i]))) return LCF_ERROR_CUDA;
    uint64_t pay;
    std::memcpy(&pay, ws->hstage + 32 * i + 24, 8);
    if (off + pay > out_capacity) return LCF_ERROR_BUFFER_TOO_SMALL;
    const uint8_t* sub = d_sub + i * sub_cap;
    if (!cuda_ok(cudaStreamWaitEvent(ws->d2h, evC[i], 0)) ||
        !cuda_ok(cudaMemcpyAsync(h_out + kHeaderBytes + 4 * c0, sub + kHeaderBytes, 4 * kc, cudaMemcpyDeviceToHost,
                                 ws->d2h)) ||
        (pay && !cuda_ok(cudaMemcpyAsync(h_out + off, sub + sbase, pay, cudaMemcpyDeviceToHost, ws->d2h))))
      return LCF_ERROR_CUDA;
    off += pay;
    return LCF_SUCCESS;
  };
  for (uint64_t i = 0; i < k; ++i) {
    const uint64_t b0 = i * sc * kChunkBytes;
    const uint64_t bytes = (b0 + sc * kChunkBytes < in_bytes ? sc * kChunkBytes : in_bytes - b0);
    if (!cuda_ok(cudaMemcpyAsync(d_in + b0, h_in + b0, bytes, cudaMemcpyHostToDevice, ws->h2d)) ||
        !cuda_ok(cudaEventRecord(evH[i], ws->h2d)) || !cuda_ok(cudaStreamWaitEvent(ws->stream, evH[i], 0)))
      return LCF_ERROR_CUDA;
    uint8_t* sub = d_sub + i * sub_cap;
    if ((st = lcf_compress(algo, dtype, d_in + b0, bytes, sub, sub_cap, nullptr, ws->stream))) return st;
    if (!cuda_ok(cudaMemcpyAsync(ws->hstage + 32 * i, sub, 32, cudaMemcpyDeviceToHost, ws->stream)) ||
        !cuda_ok(cudaEventRecord(evC[i], ws->stream)))
      return LCF_ERROR_CUDA;
    if (i >= 1 && (st = finish(i - 1))) return st;
  }
  if ((st = finish(k - 1))) return st;
  put_header(h_out, algo, in_bytes, C, off - base);
  std::memset(h_out + kHeaderBytes + 4 * C, 0, base - kHeaderBytes - 4 * C);
  if (!cuda_ok(cudaStreamSynchronize(ws->d2h))) return LCF_ERROR_CUDA;
  *out_bytes = off;
  return LCF_SUCCESS;
}

static lcf_status_t decompress_host_pipelined(lcf_algo_t algo, lcf_dtype_t dtype, const uint8_t* h_in, size_t in_bytes,
                                       uint8_t* h_out, size_t out_capacity, size_t* out_bytes, Workspace* ws,
                                       uint64_t n_bytes, uint64_t C, uint64_t payload, uint64_t sc) {
  const uint64_t k = (C + sc - 1) / sc;
  const uint64_t base = round16(kHeaderBytes + 4 * C);
  const uint32_t* table = reinterpret_cast<const uint32_t*>(h_in + kHeaderBytes);
  const uint64_t sub_hdr = round16(kHeaderBytes + 4 * sc);  // staging bytes per slice (sub-header + table + pad)
  lcf_status_t st;
  if ((st = host_pipe_init(ws, 2 * k, k * sub_hdr))) return st;
  {
    std::lock_guard<std::mutex> g(ws->mu);
    if ((st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[0]), ws->scratch_cap[0],
                   k * sub_hdr + round16(in_bytes) + 16 * k, ws->stream, false)) ||
        (st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[1]), ws->scratch_cap[1], round16(n_bytes) + 16,
                   ws->stream, false)))
      return st;
  }
  uint8_t* d_sub = static_cast<uint8_t*>(ws->scratch[0]);
  uint8_t* d_out = static_cast<uint8_t*>(ws->scratch[1]);
  cudaEvent_t* evH = ws->ev.data();
  cudaEvent_t* evC = ws->ev.data() + k;
  uint64_t off = 0, dpos = 0;  // payload offset in the stream; next free byte of d_sub
  for (uint64_t i = 0; i < k; ++i) {
    const uint64_t c0 = i * sc, kc = (c0 + sc < C ? sc : C - c0);
    uint64_t pay = 0;
    for (uint64_t c = c0; c < c0 + kc; ++c) pay += round16(table[c] & ~kRawFlag);
    if (off + pay > payload) return LCF_ERROR_CORRUPT_STREAM;
    const uint64_t b0 = c0 * kChunkBytes;
    const uint64_t bytes = (b0 + kc * kChunkBytes < n_bytes ? kc * kChunkBytes : n_bytes - b0);
    const uint64_t sbase = round16(kHeaderBytes + 4 * kc);
    uint8_t* stg = ws->hstage + i * sub_hdr;
    put_header(stg, algo, bytes, kc, pay);
    std::memcpy(stg + kHeaderBytes, table + c0, 4 * kc);
    std::memset(stg + kHeaderBytes + 4 * kc, 0, sbase - kHeaderBytes - 4 * kc);
    uint8_t* sub = d_sub + dpos;
    dpos += sbase + round16(pay);
    if (!cuda_ok(cudaMemcpyAsync(sub, stg, sbase, cudaMemcpyHostToDevice, ws->h2d)) ||
        (pay && !cuda_ok(cudaMemcpyAsync(sub + sbase, h_in + base + off, pay, cudaMemcpyHostToDevice, ws->h2d))) ||
        !cuda_ok(cudaEventRecord(evH[i], ws->h2d)) || !cuda_ok(cudaStreamWaitEvent(ws->stream, evH[i], 0)))
      return LCF_ERROR_CUDA;
    if ((st = lcf_decompress(algo, dtype, sub, sbase + pay, d_out + b0, bytes, nullptr, ws->stream))) return st;
    if (!cuda_ok(cudaEventRecord(evC[i], ws->stream)) || !cuda_ok(cudaStreamWaitEvent(ws->d2h, evC[i], 0)) ||
        !cuda_ok(cudaMemcpyAsync(h_out + b0, d_out + b0, bytes, cudaMemcpyDeviceToHost, ws->d2h)))
      return LCF_ERROR_CUDA;
    off += pay;
  }
  if (off != payload) return LCF_ERROR_CORRUPT_STREAM;
  if (!cuda_ok(cudaStreamSynchronize(ws->d2h))) return LCF_ERROR_CUDA;
  if ((st = lcf_check_stream(ws->stream))) return st;  // any slice the device found malformed
  (void)out_capacity;
  *out_bytes = n_bytes;
  return LCF_SUCCESS;
}

// DPratio decompression in tile ranges: the header and size table go up first,
// then slice i's payload bytes; the tile-range decode of slice i (DecArgs
// first_tile/end_tile/base_off) resolves FCM distances into earlier slices
// from the output they already wrote (same stream, so final), and its tiles
// come back while later slices go up and decode. Compression stays serial:
// FCM's sort needs the whole array before anything is encoded (L172).
static lcf_status_t decompress_host_dpratio_pipelined(const uint8_t* h_in, size_t in_bytes, uint8_t* h_out,
                                                      size_t* out_bytes, Workspace* ws, uint64_t n_bytes,
                                                      uint64_t C, uint64_t payload, uint64_t st_tiles) {
  const uint64_t T = C / 2, k = (T + st_tiles - 1) / st_tiles;
  const uint64_t base = round16(kHeaderBytes + 4 * C);
  const uint32_t* table = reinterpret_cast<const uint32_t*>(h_in + kHeaderBytes);
  lcf_status_t st;
  if ((st = host_pipe_init(ws, 2 * k, 16))) return st;
  {
    std::lock_guard<std::mutex> g(ws->mu);
    if ((st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[0]), ws->scratch_cap[0], round16(in_bytes) + 16,
                   ws->stream, false)) ||
        (st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[1]), ws->scratch_cap[1], round16(n_bytes) + 16,
                   ws->stream, false)) ||
        (st = grow(ws->status, ws->status_cap, C, ws->stream, true)) ||
        (st = grow(ws->tile_flag, ws->tile_cap, T + 1, ws->stream, true)))
      return st;
  }
  uint8_t* d_in = static_cast<uint8_t*>(ws->scratch[0]);
  uint8_t* d_out = static_cast<uint8_t*>(ws->scratch[1]);
  cudaEvent_t* evH = ws->ev.data();
  cudaEvent_t* evC = ws->ev.data() + k;
  if (!cuda_ok(cudaMemcpyAsync(d_in, h_in, base, cudaMemcpyHostToDevice, ws->h2d))) return LCF_ERROR_CUDA;
  uint64_t off = 0;
  for (uint64_t i = 0; i < k; ++i) {
    const uint64_t t0 = i * st_tiles, t1 = (t0 + st_tiles < T ? t0 + st_tiles : T);
    uint64_t pay = 0;
    for (uint64_t c = 2 * t0; c < 2 * t1; ++c) pay += round16(table[c] & ~kRawFlag);
    if (off + pay > payload) return LCF_ERROR_CORRUPT_STREAM;
    if ((pay && !cuda_ok(cudaMemcpyAsync(d_in + base + off, h_in + base + off, pay, cudaMemcpyHostToDevice,
                                         ws->h2d))) ||
        !cuda_ok(cudaEventRecord(evH[i], ws->h2d)) || !cuda_ok(cudaStreamWaitEvent(ws->stream, evH[i], 0)))
      return LCF_ERROR_CUDA;
    {
      std::lock_guard<std::mutex> g(ws->mu);
      DecArgs a{};
      a.stream = d_in;
      a.stream_bytes = in_bytes;
      a.out = d_out;
      a.out_capacity = n_bytes;
      a.algo = LCF_DPRATIO;
      a.word_bytes = 8;
      a.tile_flag = ws->tile_flag;
      a.first_tile = t0;
      a.end_tile = t1;
      a.base_off = off;
      LaunchCtx ctx = make_ctx(ws);
      if ((st = dpratio_decode_range(ws, a, ctx, t1 - t0, t1, ws->stream))) return st;
      ++g_launches;
      if ((st = last_launch_status())) return st;
    }
    const uint64_t b0 = t0 * 2048 * 8, b1 = (t1 * 2048 * 8 < n_bytes ? t1 * 2048 * 8 : n_bytes);
    if (!cuda_ok(cudaEventRecord(evC[i], ws->stream)) || !cuda_ok(cudaStreamWaitEvent(ws->d2h, evC[i], 0)) ||
        !cuda_ok(cudaMemcpyAsync(h_out + b0, d_out + b0, b1 - b0, cudaMemcpyDeviceToHost, ws->d2h)))
      return LCF_ERROR_CUDA;
    off += pay;
  }
  if (off != payload) return LCF_ERROR_CORRUPT_STREAM;
  if (!cuda_ok(cudaStreamSynchronize(ws->d2h))) return LCF_ERROR_CUDA;
  if ((st = lcf_check_stream(ws->stream))) return st;
  *out_bytes = n_bytes;
  return LCF_SUCCESS;
}

// DPratio compression in tile slices (the sharded-DPratio machinery, §7 of
// DESIGN.md, with slices for shards): slice i is summarised (its FCM sort),
// encoded with the carry of slices < i (the sort is reused), and the carry for
// slice i+1 = merge(carry_i, summary_i). The pieces stitch into exactly the
// lcf_compress stream, and the H2D of slice i+1, the codec on slice i and the
// D2H of slice i−1 overlap on the three streams.
static lcf_status_t compress_host_dpratio_pipelined(const uint8_t* h_in, size_t in_bytes, uint8_t* h_out,
                                                    size_t out_capacity, size_t* out_bytes, Workspace* ws,
                                                    uint64_t st_tiles) {
  const uint64_t n = in_bytes / 8, T = (n + 2047) / 2048, k = (T + st_tiles - 1) / st_tiles;
  const uint64_t C = 2 * T, base = round16(kHeaderBytes + 4 * C);
  if (out_capacity < base) return LCF_ERROR_BUFFER_TOO_SMALL;
  const size_t sb = lcf_dpratio_summary_bytes();
  const uint64_t slice_words = st_tiles * 2048;
  const size_t piece_cap = round16(4 * 2 * st_tiles) + payload_bound(LCF_DPRATIO, 8 * slice_words) + 16;
  lcf_status_t st;
  if ((st = host_pipe_init(ws, 2 * k, 8 * k))) return st;
  {
    std::lock_guard<std::mutex> g(ws->mu);
    if ((st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[0]), ws->scratch_cap[0], round16(in_bytes) + 16,
                   ws->stream, false)) ||
        (st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[1]), ws->scratch_cap[1], k * piece_cap, ws->stream,
                   false)) ||
        (st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[3]), ws->scratch_cap[3], 4 * sb, ws->stream, false)))
      return st;
  }
  uint8_t* d_in = static_cast<uint8_t*>(ws->scratch[0]);
  uint8_t* d_pieces = static_cast<uint8_t*>(ws->scratch[1]);
  uint8_t* P[2] = {static_cast<uint8_t*>(ws->scratch[3]), static_cast<uint8_t*>(ws->scratch[3]) + 2 * sb};
  // (P[j] = carry ‖ summary, contiguous for the 2-summary merge)
  cudaEvent_t* evH = ws->ev.data();
  cudaEvent_t* evC = ws->ev.data() + k;
  uint64_t* cnt_h = reinterpret_cast<uint64_t*>(ws->hstage);
  if (!fcm_empty_carry(P[0], ws->stream)) return LCF_ERROR_CUDA;  // slice 0 has no earlier slices
  uint64_t off = base;
  auto finish = [&](uint64_t i) -> lcf_status_t {
    const uint64_t t0 = i * st_tiles, nt = (t0 + st_tiles < T ? st_tiles : T - t0);
    if (!cuda_ok(cudaEventSynchronize(evC[i]))) return LCF_ERROR_CUDA;
    const uint64_t pay = cnt_h[i];
    if (off + pay > out_capacity) return LCF_ERROR_BUFFER_TOO_SMALL;
    const uint8_t* piece = d_pieces + i * piece_cap;
    if (!cuda_ok(cudaStreamWaitEvent(ws->d2h, evC[i], 0)) ||
        !cuda_ok(cudaMemcpyAsync(h_out + kHeaderBytes + 4 * 2 * t0, piece, 4 * 2 * nt, cudaMemcpyDeviceToHost,
                                 ws->d2h)) ||
        (pay && !cuda_ok(cudaMemcpyAsync(h_out + off, piece + round16(4 * 2 * st_tiles), pay,
                                         cudaMemcpyDeviceToHost, ws->d2h))))
      return LCF_ERROR_CUDA;
    off += pay;
    return LCF_SUCCESS;
  };
  for (uint64_t i = 0; i < k; ++i) {
    const uint64_t w0 = i * slice_words, w1 = (w0 + slice_words < n ? w0 + slice_words : n);
    const uint64_t b0 = 8 * w0, bytes = 8 * (w1 - w0);
    if (!cuda_ok(cudaMemcpyAsync(d_in + b0, h_in + b0, bytes, cudaMemcpyHostToDevice, ws->h2d)) ||
        !cuda_ok(cudaEventRecord(evH[i], ws->h2d)) || !cuda_ok(cudaStreamWaitEvent(ws->stream, evH[i], 0)))
      return LCF_ERROR_CUDA;
    uint8_t* cur = P[i & 1];  // carry_i ‖ summary_i
    uint8_t* piece = d_pieces + i * piece_cap;
    uint64_t* d_cnt = reinterpret_cast<uint64_t*>(piece + piece_cap - 16);
    if ((st = lcf_dpratio_shard_summary(d_in + b0, bytes, in_bytes, w0, cur + sb, ws->stream)) ||
        (st = lcf_dpratio_compress_shard(d_in + b0, bytes, in_bytes, w0, i ? cur : nullptr, piece,
                                         piece + round16(4 * 2 * st_tiles), piece_cap - 16 - round16(4 * 2 * st_tiles),
                                         d_cnt, ws->stream)))
      return st;
    if (i + 1 < k && (st = lcf_dpratio_merge_summaries(cur, 2, P[(i + 1) & 1], ws->stream))) return st;
    if (!cuda_ok(cudaMemcpyAsync(cnt_h + i, d_cnt, 8, cudaMemcpyDeviceToHost, ws->stream)) ||
        !cuda_ok(cudaEventRecord(evC[i], ws->stream)))
      return LCF_ERROR_CUDA;
    if (i >= 1 && (st = finish(i - 1))) return st;
  }
  if ((st = finish(k - 1))) return st;
  put_header(h_out, LCF_DPRATIO, in_bytes, C, off - base);
  std::memset(h_out + kHeaderBytes + 4 * C, 0, base - kHeaderBytes - 4 * C);
  if (!cuda_ok(cudaStreamSynchronize(ws->d2h))) return LCF_ERROR_CUDA;
  *out_bytes = off;
  return LCF_SUCCESS;
}

// A failed pipelined call still has copies and kernels in flight on the
// caller's buffers: drain all three streams before reporting, and consume the
// device error word (slices already enqueued may have flagged too — this call
// reports one status, like every synchronising call).
static lcf_status_t host_pipe_done(Workspace* ws, lcf_status_t st) {
  if (st) {
    cudaStreamSynchronize(ws->h2d);
    cudaStreamSynchronize(ws->d2h);
    lcf_check_stream(ws->stream);
  }
  return st;
}

static lcf_status_t host_roundtrip(bool compress, lcf_algo_t algo, lcf_dtype_t dtype, const void* h_in,
                                   size_t in_bytes, void* h_out, size_t out_capacity, size_t* out_bytes,
                                   cudaStream_t stream) {
  if (!valid_algo(algo)) return LCF_ERROR_INVALID_ARGUMENT;
  if (!out_bytes || (in_bytes && !h_in)) return LCF_ERROR_INVALID_ARGUMENT;
  lcf_status_t st = LCF_SUCCESS;
  Workspace* ws = get_ws(stream, &st);
  if (!ws) return st;
  if (algo == LCF_DPRATIO && dtype_matches(algo, dtype) && compress && in_bytes % 8 == 0 &&
      in_bytes / 8 < (1ull << 31)) {
    std::lock_guard<std::mutex> hg(ws->host_mu);
    const uint64_t T = (in_bytes / 8 + 2047) / 2048;
    const uint64_t st_tiles = host_slice_chunks(T);
    if (T > st_tiles)
      return host_pipe_done(ws, compress_host_dpratio_pipelined(static_cast<const uint8_t*>(h_in), in_bytes,
                                                                static_cast<uint8_t*>(h_out), out_capacity, out_bytes,
                                                                ws, st_tiles));
  }
  if (algo == LCF_DPRATIO && dtype_matches(algo, dtype) && !compress && in_bytes >= kHeaderBytes) {
    std::lock_guard<std::mutex> hg(ws->host_mu);
    uint64_t nb, C, pay;
    if (lcf_status_t s = check_header(static_cast<const uint8_t*>(h_in), in_bytes, algo, &nb, &C, &pay)) return s;
    if (nb > out_capacity) return LCF_ERROR_BUFFER_TOO_SMALL;
    const uint64_t st_tiles = host_slice_chunks(C / 2);  // a tile decodes to one 16 KiB chunk of words
    if (C / 2 > st_tiles)
      return host_pipe_done(ws, decompress_host_dpratio_pipelined(static_cast<const uint8_t*>(h_in), in_bytes,
                                                                  static_cast<uint8_t*>(h_out), out_bytes, ws, nb,
                                                                  C, pay, st_tiles));
  }
  if (algo != LCF_DPRATIO && dtype_matches(algo, dtype)) {  // pipelined slices (chunk-local codecs)
    std::lock_guard<std::mutex> hg(ws->host_mu);
    if (compress) {
      const uint64_t C = lcf_num_chunks(algo, in_bytes);
      const uint64_t sc = host_slice_chunks(C);
      if (in_bytes % word_bytes_of(algo) == 0 && C > sc)
        return host_pipe_done(ws, compress_host_pipelined(algo, dtype, static_cast<const uint8_t*>(h_in), in_bytes,
                                                          static_cast<uint8_t*>(h_out), out_capacity, out_bytes,
                                                          ws, C, sc));
    } else if (in_bytes >= kHeaderBytes) {
      uint64_t nb, C, pay;
      if (lcf_status_t s = check_header(static_cast<const uint8_t*>(h_in), in_bytes, algo, &nb, &C, &pay)) return s;
      if (nb > out_capacity) return LCF_ERROR_BUFFER_TOO_SMALL;
      const uint64_t sc = host_slice_chunks(C);
      if (C > sc)
        return host_pipe_done(ws, decompress_host_pipelined(algo, dtype, static_cast<const uint8_t*>(h_in),
                                                            in_bytes, static_cast<uint8_t*>(h_out), out_capacity,
                                                            out_bytes, ws, nb, C, pay, sc));
    }
  }
  size_t dcap;
  if (compress) {
    dcap = lcf_max_compressed_size(algo, dtype, in_bytes);
  } else {
    if (in_bytes < 32) return LCF_ERROR_CORRUPT_STREAM;
    uint64_t nb;
    std::memcpy(&nb, static_cast<const uint8_t*>(h_in) + 8, 8);
    if (nb > out_capacity) return LCF_ERROR_BUFFER_TOO_SMALL;
    dcap = nb;
  }
  {
    std::lock_guard<std::mutex> g(ws->mu);
    if ((st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[0]), ws->scratch_cap[0], round16(in_bytes) + 16, stream, false)))
      return st;
    if ((st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[1]), ws->scratch_cap[1], round16(dcap) + 16, stream, false)))
      return st;
    if (!cuda_ok(cudaMemcpyAsync(ws->scratch[0], h_in, in_bytes, cudaMemcpyHostToDevice, stream)))
      return LCF_ERROR_CUDA;
  }
  size_t n = 0;
  st = compress ? lcf_compress(algo, dtype, ws->scratch[0], in_bytes, ws->scratch[1], dcap, &n, stream)
                : lcf_decompress(algo, dtype, ws->scratch[0], in_bytes, ws->scratch[1], dcap, &n, stream);
  if (st) return st;
  if (n > out_capacity) return LCF_ERROR_BUFFER_TOO_SMALL;
  if (!cuda_ok(cudaMemcpyAsync(h_out, ws->scratch[1], n, cudaMemcpyDeviceToHost, stream)) ||
      !cuda_ok(cudaStreamSynchronize(stream)))
    return LCF_ERROR_CUDA;
  *out_bytes = n;
  return LCF_SUCCESS;
}

lcf_status_t lcf_compress_host(lcf_algo_t algo, lcf_dtype_t dtype, const void* h_in, size_t in_bytes, void* h_out,
                               size_t out_capacity, size_t* out_bytes, void* stream) {
  return host_roundtrip(true, algo, dtype, h_in, in_bytes, h_out, out_capacity, out_bytes, (cudaStream_t)stream);
}
lcf_status_t lcf_decompress_host(lcf_algo_t algo, lcf_dtype_t dtype, const void* h_in, size_t in_bytes, void* h_out,
                                 size_t out_capacity, size_t* out_bytes, void* stream) {
  return host_roundtrip(false, algo, dtype, h_in, in_bytes, h_out, out_capacity, out_bytes, (cudaStream_t)stream);
}

lcf_status_t lcf_compress_shard(lcf_algo_t algo, lcf_dtype_t dtype, const void* d_in_shard, size_t shard_bytes,
                                size_t total_in_bytes, uint64_t first_chunk, void* d_table_slice, void* d_payload,
                                size_t payload_capacity, uint64_t* d_payload_bytes, void* stream_) {
  cudaStream_t stream = (cudaStream_t)stream_;
  if (!valid_algo(algo) || algo == LCF_DPRATIO) return LCF_ERROR_INVALID_ARGUMENT;
  if (!dtype_matches(algo, dtype)) return LCF_ERROR_DTYPE_MISMATCH;
  const uint32_t wb = word_bytes_of(algo);
  if (total_in_bytes % wb || shard_bytes % wb || !d_payload_bytes) return LCF_ERROR_INVALID_ARGUMENT;
  const uint64_t C = lcf_num_chunks(algo, total_in_bytes);
  if (first_chunk > C || first_chunk * kChunkBytes + shard_bytes > total_in_bytes) return LCF_ERROR_INVALID_ARGUMENT;
  const bool has_tail = first_chunk * kChunkBytes + shard_bytes == total_in_bytes;
  if (!has_tail && shard_bytes % kChunkBytes) return LCF_ERROR_INVALID_ARGUMENT;
  const uint64_t k = (shard_bytes + kChunkBytes - 1) / kChunkBytes;
  if (k && (!d_in_shard || !aligned16(d_in_shard) || !d_table_slice || !d_payload || !aligned16(d_payload)))
    return LCF_ERROR_INVALID_ARGUMENT;
  if (payload_capacity < (shard_bytes / kChunkBytes) * kChunkBytes + round16(shard_bytes % kChunkBytes))
    return LCF_ERROR_BUFFER_TOO_SMALL;
  lcf_status_t st = LCF_SUCCESS;
  Workspace* ws = get_ws(stream, &st);
  if (!ws) return st;
  std::lock_guard<std::mutex> g(ws->mu);
  if (k == 0) return cuda_ok(cudaMemsetAsync(d_payload_bytes, 0, 8, stream)) ? LCF_SUCCESS : LCF_ERROR_CUDA;
  EncArgs a = enc_args(algo, d_in_shard, total_in_bytes);
  a.first_chunk = first_chunk;
  a.n_chunks = k;
  a.stream_chunks = C;
  a.table = static_cast<uint32_t*>(d_table_slice);
  a.payload = static_cast<uint8_t*>(d_payload);
  a.count_out = d_payload_bytes;
  return enqueue_encode(ws, a);
}

size_t lcf_dpratio_summary_bytes(void) { return fcm_carry_bytes(); }

// Validation shared by the sharded DPratio calls: whole tiles, in range.
static lcf_status_t dp_shard_args(const void* d_x, size_t shard_bytes, size_t total_in_bytes, uint64_t first_word) {
  if (total_in_bytes % 8 || shard_bytes % 8 || first_word % 2048) return LCF_ERROR_INVALID_ARGUMENT;
  if (total_in_bytes / 8 >= (1ull << 31)) return LCF_ERROR_INVALID_ARGUMENT;  // 32-bit FCM indices
  if (first_word * 8 + shard_bytes > total_in_bytes) return LCF_ERROR_INVALID_ARGUMENT;
  if (first_word * 8 + shard_bytes != total_in_bytes && shard_bytes % kChunkBytes) return LCF_ERROR_INVALID_ARGUMENT;
  if (shard_bytes && (!d_x || (reinterpret_cast<uintptr_t>(d_x) & 15))) return LCF_ERROR_INVALID_ARGUMENT;
  return LCF_SUCCESS;
}

lcf_status_t lcf_dpratio_shard_summary(const void* d_x, size_t shard_bytes, size_t total_in_bytes, uint64_t first_word,
                                       void* d_summary, void* stream_) {
  cudaStream_t stream = (cudaStream_t)stream_;
  if (lcf_status_t s = dp_shard_args(d_x, shard_bytes, total_in_bytes, first_word)) return s;
  if (!d_summary) return LCF_ERROR_INVALID_ARGUMENT;
  lcf_status_t st = LCF_SUCCESS;
  Workspace* ws = get_ws(stream, &st);
  if (!ws) return st;
  std::lock_guard<std::mutex> g(ws->mu);
  const uint64_t n = shard_bytes / 8;
  if ((st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[2]), ws->scratch_cap[2], dpratio_fcm_workspace(n), stream,
                 false)))
    return st;
  uint32_t* dist = nullptr;
  g_launches += launch_fcm_shard(static_cast<const uint64_t*>(d_x), n, (uint32_t)(first_word < 3 ? first_word : 3),
                                 first_word, nullptr, d_summary, false, ws->scratch[2], ws->scratch_cap[2], stream,
                                 &dist);
  if ((st = last_launch_status())) return st;
  ws->sorted_x = d_x;
  ws->sorted_ws = ws->scratch[2];
  ws->sorted_n = n;
  ws->sorted_first = first_word;
  return LCF_SUCCESS;
}

lcf_status_t lcf_dpratio_merge_summary_ptrs(const void* const* d_summaries, size_t count, void* d_carry,
                                            void* stream_) {
  cudaStream_t stream = (cudaStream_t)stream_;
  if (!d_carry || (count && !d_summaries) || count > 64) return LCF_ERROR_INVALID_ARGUMENT;
  for (size_t r = 0; r < count; ++r)
    if (!d_summaries[r]) return LCF_ERROR_INVALID_ARGUMENT;
  g_launches += launch_fcm_carry_merge(d_summaries, (uint32_t)count, d_carry, stream);
  return last_launch_status();
}

lcf_status_t lcf_dpratio_merge_summaries(const void* d_summaries, size_t count, void* d_carry, void* stream) {
  if (!d_carry || (count && !d_summaries) || count > 64) return LCF_ERROR_INVALID_ARGUMENT;
  const void* p[64];
  for (size_t r = 0; r < count; ++r) p[r] = static_cast<const uint8_t*>(d_summaries) + r * fcm_carry_bytes();
  return lcf_dpratio_merge_summary_ptrs(p, count, d_carry, stream);
}

// ---- CUDA IPC plumbing (include/lcf.h) ---------------------------------------
// The export handle covers the whole allocation holding d_ptr (found with the
// driver's cuMemGetAddressRange, fetched at run time so that the library
// needs no link-time libcuda); the importer adds the offset back.
namespace {
typedef int (*AddrRangeFn)(unsigned long long*, size_t*, unsigned long long);
std::mutex g_ipc_mu;
// several tensors of one peer allocation map it once (the driver maps a
// handle once per process): handle bytes → (base, imports); pointer → handle
std::map<std::string, std::pair<void*, int>> g_ipc_maps;
std::multimap<void*, std::string> g_ipc_ptrs;
}  // namespace

lcf_status_t lcf_ipc_export(const void* d_ptr, void* handle64, uint64_t* offset) {
  if (!d_ptr || !handle64 || !offset) return LCF_ERROR_INVALID_ARGUMENT;
  static AddrRangeFn range = [] {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      fn = nullptr;
    return reinterpret_cast<AddrRangeFn>(fn);
  }();
  if (!range) return LCF_ERROR_CUDA;
  unsigned long long base = 0;
  size_t size = 0;
  if (range(&base, &size, (unsigned long long)(uintptr_t)d_ptr) != 0) return LCF_ERROR_INVALID_ARGUMENT;
  cudaIpcMemHandle_t h;
  if (!cuda_ok(cudaIpcGetMemHandle(&h, reinterpret_cast<void*>(base)))) return LCF_ERROR_CUDA;
  static_assert(sizeof(h) == 64, "64-byte IPC handle");
  memcpy(handle64, &h, 64);
  *offset = (uint64_t)((uintptr_t)d_ptr - base);
  return LCF_SUCCESS;
}

lcf_status_t lcf_ipc_import(const void* handle64, uint64_t offset, void** d_ptr) {
  if (!handle64 || !d_ptr) return LCF_ERROR_INVALID_ARGUMENT;
  const std::string key(static_cast<const char*>(handle64), 64);
  std::lock_guard<std::mutex> g(g_ipc_mu);
  auto it = g_ipc_maps.find(key);
  if (it == g_ipc_maps.end()) {
    cudaIpcMemHandle_t h;
    memcpy(&h, handle64, 64);
    void* base = nullptr;
    if (!cuda_ok(cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess))) return LCF_ERROR_CUDA;
    it = g_ipc_maps.emplace(key, std::make_pair(base, 0)).first;
  }
  ++it->second.second;
  *d_ptr = static_cast<uint8_t*>(it->second.first) + offset;
  g_ipc_ptrs.emplace(*d_ptr, key);
  return LCF_SUCCESS;
}

lcf_status_t lcf_ipc_close(void* d_ptr) {
  std::lock_guard<std::mutex> g(g_ipc_mu);
  auto p = g_ipc_ptrs.find(d_ptr);
  if (p == g_ipc_ptrs.end()) return LCF_ERROR_INVALID_ARGUMENT;
  auto it = g_ipc_maps.find(p->second);
  g_ipc_ptrs.erase(p);
  if (--it->second.second > 0) return LCF_SUCCESS;
  void* base = it->second.first;
  g_ipc_maps.erase(it);
  return cuda_ok(cudaIpcCloseMemHandle(base)) ? LCF_SUCCESS : LCF_ERROR_CUDA;
}

lcf_status_t lcf_dpratio_compress_shard(const void* d_x, size_t shard_bytes, size_t total_in_bytes,
                                        uint64_t first_word, const void* d_carry, void* d_table_slice,
                                        void* d_payload, size_t payload_capacity, uint64_t* d_payload_bytes,
                                        void* stream_) {
  cudaStream_t stream = (cudaStream_t)stream_;
  if (lcf_status_t s = dp_shard_args(d_x, shard_bytes, total_in_bytes, first_word)) return s;
  if (!d_payload_bytes) return LCF_ERROR_INVALID_ARGUMENT;
  const uint64_t n = shard_bytes / 8, tiles = (n + 2047) / 2048;
  if (tiles && (!d_table_slice || !d_payload || !aligned16(d_payload))) return LCF_ERROR_INVALID_ARGUMENT;
  if (payload_capacity < payload_bound(LCF_DPRATIO, shard_bytes)) return LCF_ERROR_BUFFER_TOO_SMALL;
  lcf_status_t st = LCF_SUCCESS;
  Workspace* ws = get_ws(stream, &st);
  if (!ws) return st;
  std::lock_guard<std::mutex> g(ws->mu);
  if (tiles == 0) return cuda_ok(cudaMemsetAsync(d_payload_bytes, 0, 8, stream)) ? LCF_SUCCESS : LCF_ERROR_CUDA;
  EncArgs a = enc_args(LCF_DPRATIO, d_x, shard_bytes);  // the shard's words; tiles of the launch from 0
  a.first_chunk = 2 * (first_word / 2048);
  a.n_chunks = 2 * tiles;
  a.stream_chunks = lcf_num_chunks(LCF_DPRATIO, total_in_bytes);
  a.table = static_cast<uint32_t*>(d_table_slice);
  a.payload = static_cast<uint8_t*>(d_payload);
  a.count_out = d_payload_bytes;
  if ((st = grow(ws->status, ws->status_cap, a.n_chunks, stream, true)) ||
      (st = grow(reinterpret_cast<uint8_t*&>(ws->scratch[2]), ws->scratch_cap[2], dpratio_fcm_workspace(n), stream,
                 false)))
    return st;
  // the summary call on this stream already sorted this shard: skip the sort
  const bool sorted = ws->sorted_x == d_x && ws->sorted_ws == ws->scratch[2] && ws->sorted_n == n &&
                      ws->sorted_first == first_word;
  ws->sorted_x = nullptr;
  LaunchCtx ctx = make_ctx(ws);
  g_launches += launch_dpratio_encode(a, ctx, ws->scratch[2], ws->scratch_cap[2], stream,
                                      (uint32_t)(first_word < 3 ? first_word : 3), first_word, d_carry, sorted);
  return last_launch_status();
}

lcf_status_t lcf_dpratio_decompress_shard(const void* d_in, size_t in_bytes, uint64_t first_word, void* d_out,
                                          size_t out_capacity, uint32_t* d_pending, void* stream_) {
  cudaStream_t stream = (cudaStream_t)stream_;
  if (!d_in || !aligned16(d_in) || !d_pending || (out_capacity && (!d_out || !aligned16(d_out))))
    return LCF_ERROR_INVALID_ARGUMENT;
  if (first_word % 2048) return LCF_ERROR_INVALID_ARGUMENT;
  if (in_bytes < kHeaderBytes) return LCF_ERROR_CORRUPT_STREAM;
  lcf_status_t st = LCF_SUCCESS;
  Workspace* ws = get_ws(stream, &st);
  if (!ws) return st;
  std::lock_guard<std::mutex> g(ws->mu);
  const uint64_t by_table = (in_bytes - kHeaderBytes) / 4;
  const uint64_t by_out = 2 * ((out_capacity + kChunkBytes - 1) / kChunkBytes);
  uint64_t grid = by_table < by_out ? by_table : by_out;
  if (grid == 0) grid = 1;
  if ((st = grow(ws->status, ws->status_cap, grid, stream, true)) ||
      (st = grow(ws->tile_flag, ws->tile_cap, grid / 2 + 1, stream, true)))
    return st;
  const uint64_t W = (out_capacity / 8 + 31) / 32;  // d_pending: pending bits ‖ chain-node marks
  if (!cuda_ok(cudaMemsetAsync(d_pending, 0, 2 * 4 * W, stream))) return LCF_ERROR_CUDA;
  DecArgs a{};
  a.stream = static_cast<const uint8_t*>(d_in);
  a.stream_bytes = in_bytes;
  a.out = static_cast<uint8_t*>(d_out);
  a.out_capacity = out_capacity;
  a.algo = LCF_DPRATIO;
  a.word_bytes = 8;
  a.tile_flag = ws->tile_flag;
  a.gbase = first_word;
  a.pend = d_pending;
  a.tgt = d_pending + W;
  a.any_pend = ws->any_pend;
  LaunchCtx ctx = make_ctx(ws);
  launch_dpratio_decode(a, ctx, grid / 2 + 1, stream);
  ++g_launches;
  return last_launch_status();
}

// The views of lcf_dpratio_find_roots / gather_roots (include/lcf.h).
static lcf_status_t dp_views(const lcf_dp_view* views, size_t count, size_t self, DpViews& v) {
  if (!views || count == 0 || count > kMaxViews || self >= count) return LCF_ERROR_INVALID_ARGUMENT;
  v.count = (uint32_t)count;
  v.self = (uint32_t)self;
  for (size_t q = 0; q < count; ++q) {
    const lcf_dp_view& w = views[q];
    if (q ? w.first_word != views[q - 1].first_word + views[q - 1].n_words : w.first_word != 0)
      return LCF_ERROR_INVALID_ARGUMENT;  // sorted, contiguous from word 0
    if (w.n_words && (!w.d_words || !w.d_pending)) return LCF_ERROR_INVALID_ARGUMENT;
    v.v[q] = DpView{w.first_word, w.n_words, static_cast<uint64_t*>(w.d_words), w.d_pending,
                    w.d_pending + (w.n_words + 31) / 32};
  }
  if (views[self].first_word % 32) return LCF_ERROR_INVALID_ARGUMENT;
  return LCF_SUCCESS;
}

static lcf_status_t dp_roots(const lcf_dp_view* views, size_t count, size_t self, void* stream_, bool gather) {
  cudaStream_t stream = (cudaStream_t)stream_;
  DpViews v{};
  if (lcf_status_t s = dp_views(views, count, self, v)) return s;
  lcf_status_t st = LCF_SUCCESS;
  Workspace* ws = get_ws(stream, &st);
  if (!ws) return st;
  std::lock_guard<std::mutex> g(ws->mu);
  LaunchCtx ctx = make_ctx(ws);
  const uint64_t n = views[self].n_words;
  if (gather) {
    launch_dp_gather_roots(v, nullptr, 0, n, ctx, nullptr, stream);
    if (n) ++g_launches;
  } else {
    launch_dp_find_roots(v, nullptr, 0, n, ctx, nullptr, stream, 0);  // chain nodes first
    launch_dp_find_roots(v, nullptr, 0, n, ctx, nullptr, stream, 1);
    if (n) g_launches += 2;
  }
  return last_launch_status();
}

lcf_status_t lcf_dpratio_find_roots(const lcf_dp_view* views, size_t count, size_t self, void* stream) {
  return dp_roots(views, count, self, stream, false);
}

lcf_status_t lcf_dpratio_gather_roots(const lcf_dp_view* views, size_t count, size_t self, void* stream) {
  return dp_roots(views, count, self, stream, true);
}

lcf_status_t lcf_write_header(lcf_algo_t algo, lcf_dtype_t dtype, size_t total_in_bytes,
                              uint64_t total_payload_bytes, void* d_stream, void* stream_) {
  if (!valid_algo(algo)) return LCF_ERROR_INVALID_ARGUMENT;
  if (!dtype_matches(algo, dtype)) return LCF_ERROR_DTYPE_MISMATCH;
  if (!d_stream || !aligned16(d_stream) || total_in_bytes % word_bytes_of(algo)) return LCF_ERROR_INVALID_ARGUMENT;
  const uint64_t C = lcf_num_chunks(algo, total_in_bytes);
  const uint64_t base = round16(kHeaderBytes + 4 * C);
  EncArgs a = enc_args(algo, nullptr, total_in_bytes);
  a.stream_chunks = C;
  a.header = reinterpret_cast<StreamHeader*>(d_stream);
  a.pad_start = static_cast<uint8_t*>(d_stream) + kHeaderBytes + 4 * C;
  a.pad_len = (uint32_t)(base - kHeaderBytes - 4 * C);
  a.payload_total = total_payload_bytes;
  launch_write_header(a, (cudaStream_t)stream_);
  ++g_launches;
  return last_launch_status();
}

}  // extern "C"
