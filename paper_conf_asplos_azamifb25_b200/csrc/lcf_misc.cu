// lcf_misc.cu — stream header writer (FORMAT.md §1) for empty inputs and for
// the sharded mode (lcf_write_header), where no chunk CTA writes it.
#include "lcf_kernels.cuh"

namespace lcf {
namespace {
__global__ void write_header_kernel(EncArgs a) {
  if (threadIdx.x == 0) finish_encode(a, a.payload_total);
  if (threadIdx.x < a.pad_len) a.pad_start[threadIdx.x] = 0;
}
}  // namespace

void launch_write_header(const EncArgs& a, cudaStream_t st) {
  EncArgs b = a;
  b.count_out = nullptr;
  KTrace kt("write_header", st);
  write_header_kernel<<<1, 32, 0, st>>>(b);
}
}  // namespace lcf

// ---- kernel-time tracing (lcf_profile_enable / lcf_profile_report) ------------
#include <lcf.h>

#include <map>
#include <mutex>
#include <string>
#include <vector>

namespace {
struct TraceRec {
  const char* name;
  cudaEvent_t a, b;
};
std::mutex g_trace_mu;
bool g_trace_on = false;
std::vector<TraceRec> g_trace;
}  // namespace

namespace lcf {
KTrace::KTrace(const char* n, cudaStream_t s) : name(n), st(s), rec(nullptr) {
  if (!g_trace_on) return;
  auto* r = new TraceRec{n, nullptr, nullptr};
  cudaEventCreate(&r->a);
  cudaEventCreate(&r->b);
  cudaEventRecord(r->a, s);
  rec = r;
}
KTrace::~KTrace() {
  if (!rec) return;
  auto* r = static_cast<TraceRec*>(rec);
  cudaEventRecord(r->b, st);
  std::lock_guard<std::mutex> g(g_trace_mu);
  g_trace.push_back(*r);
  delete r;
}
}  // namespace lcf

extern "C" {
void lcf_profile_enable(int enable) {
  std::lock_guard<std::mutex> g(g_trace_mu);
  g_trace_on = enable != 0;
}

size_t lcf_profile_report(char* buf, size_t cap) {
  std::vector<TraceRec> recs;
  {
    std::lock_guard<std::mutex> g(g_trace_mu);
    recs.swap(g_trace);
  }
  std::map<std::string, std::pair<unsigned, double>> agg;
  for (auto& r : recs) {
    cudaEventSynchronize(r.b);
    float ms = 0;
    cudaEventElapsedTime(&ms, r.a, r.b);
    auto& e = agg[r.name];
    e.first += 1;
    e.second += ms;
    cudaEventDestroy(r.a);
    cudaEventDestroy(r.b);
  }
  std::string out;
  for (auto& kv : agg)
    out += kv.first + " " + std::to_string(kv.second.first) + " " + std::to_string(kv.second.second) + "\n";
  if (buf && cap) {
    const size_t n = out.size() < cap - 1 ? out.size() : cap - 1;
    out.copy(buf, n);
    buf[n] = 0;
  }
  return out.size();
}
}
