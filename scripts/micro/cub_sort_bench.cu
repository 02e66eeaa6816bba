// Micro-benchmark: CUB radix sort variants for FCM-sized inputs (37.7 M pairs,
// 20-bit keys). Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o cub_sort_bench cub_sort_bench.cu
#include <cub/cub.cuh>
#include <cstdio>
#include <vector>
__global__ void fill(uint32_t* k, uint64_t* v, uint32_t* v32, uint64_t* k64, int n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    uint64_t h = (uint64_t)i * 0x9E3779B97F4A7C15ull;
    k[i] = (uint32_t)(h >> 44);
    v[i] = ((uint64_t)(uint32_t)(h ^ 1234567) << 32) | (uint32_t)i;
    v32[i] = i;
    k64[i] = ((uint64_t)k[i] << 32) | (uint32_t)i;
  }
}
template <class F> float timeit(F f) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  f(); cudaDeviceSynchronize();
  float best = 1e9;
  for (int r = 0; r < 5; ++r) { cudaEventRecord(a); f(); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); best = ms < best ? ms : best; }
  return best;
}
int main() {
  const int n = 37748736;
  uint32_t *k, *k2, *v32, *v32b; uint64_t *v, *v2, *k64, *k64b;
  cudaMalloc(&k, 4ull * n); cudaMalloc(&k2, 4ull * n); cudaMalloc(&v, 8ull * n); cudaMalloc(&v2, 8ull * n);
  cudaMalloc(&v32, 4ull * n); cudaMalloc(&v32b, 4ull * n); cudaMalloc(&k64, 8ull * n); cudaMalloc(&k64b, 8ull * n);
  fill<<<1184, 256>>>(k, v, v32, k64, n);
  size_t t1 = 0, t2 = 0, t3 = 0, t4 = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, t1, k, k2, v, v2, n, 0, 20);
  cub::DeviceRadixSort::SortPairs(nullptr, t2, k, k2, v32, v32b, n, 0, 20);
  cub::DeviceRadixSort::SortKeys(nullptr, t3, k, k2, n, 0, 20);
  cub::DeviceRadixSort::SortKeys(nullptr, t4, k64, k64b, n, 0, 52);
  size_t tm = std::max(std::max(t1, t2), std::max(t3, t4));
  void* tmp; cudaMalloc(&tmp, tm);
  printf("pairs u32/u64 20b: %.3f ms\n", timeit([&] { cub::DeviceRadixSort::SortPairs(tmp, t1, k, k2, v, v2, n, 0, 20); }));
  printf("pairs u32/u32 20b: %.3f ms\n", timeit([&] { cub::DeviceRadixSort::SortPairs(tmp, t2, k, k2, v32, v32b, n, 0, 20); }));
  printf("keys  u32     20b: %.3f ms\n", timeit([&] { cub::DeviceRadixSort::SortKeys(tmp, t3, k, k2, n, 0, 20); }));
  printf("keys  u64     52b: %.3f ms\n", timeit([&] { cub::DeviceRadixSort::SortKeys(tmp, t4, k64, k64b, n, 0, 52); }));
  {
    cub::DoubleBuffer<uint32_t> dk(k, k2);
    cub::DoubleBuffer<uint64_t> dv(v, v2);
    size_t t5 = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, t5, dk, dv, n, 0, 20);
    void* tmp5; cudaMalloc(&tmp5, t5);
    printf("pairs u32/u64 20b DoubleBuffer: %.3f ms (temp %zu MB)\n", timeit([&] { cub::DoubleBuffer<uint32_t> a(k, k2); cub::DoubleBuffer<uint64_t> b(v, v2); cub::DeviceRadixSort::SortPairs(tmp5, t5, a, b, n, 0, 20); }), t5 >> 20);
    for (int nn : {1 << 20, 4 << 20, 16 << 20}) {
      printf("pairs u32/u64 20b n=%d: %.3f ms\n", nn, timeit([&] { cub::DeviceRadixSort::SortPairs(tmp, t1, k, k2, v, v2, nn, 0, 20); }));
    }
  }
  printf("memcpy 12n bytes: %.3f ms\n", timeit([&] { cudaMemcpyAsync(v2, v, 8ull * n, cudaMemcpyDeviceToDevice); cudaMemcpyAsync(k2, k, 4ull*n, cudaMemcpyDeviceToDevice); }));
  return 0;
}
