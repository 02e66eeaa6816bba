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
  write_header_kernel<<<1, 32, 0, st>>>(b);
}
}  // namespace lcf
