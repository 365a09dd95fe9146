// tools/sorted_probe.cu — does issuing a burst of random host rows in ADDRESS order help
// (page-walk caches, DRAM locality) compared with random order?  One burst of R rows of
// 256 B over an 8 GiB mapped pinned buffer, rows given as an explicit list.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <random>
#include <vector>

#include "kernels.cuh"

__global__ void __launch_bounds__(128) list_probe(const float* host, const uint64_t* rows, int64_t n, float* sink) {
  const int lane = threadIdx.x & 31;
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g - lane >= n) return;
  const bool active = g < n;
  const float* src = active ? host + rows[g] * 64 : nullptr;
  float* dst = active ? sink + (size_t)(g & 4095) * 64 : nullptr;
  fl::gather_rows<64>(src, dst, lane);
}

int main() {
  cudaSetDevice(0);
  const size_t span = 8ull << 30;
  void* h;
  cudaHostAlloc(&h, span, cudaHostAllocMapped);
  cudaMemset(h, 1, span);
  void* d;
  cudaHostGetDevicePointer(&d, h, 0);
  float* sink;
  cudaMalloc(&sink, 4096 * 256);
  uint64_t* drows;
  cudaMalloc(&drows, 8 * (1 << 20));
  std::mt19937_64 rng(7);
  printf("{");
  for (int64_t n : {2048, 8192, 32768}) {
    for (int sorted = 0; sorted < 3; ++sorted) {
      double best = 1e30;
      for (int rep = 0; rep < 5; ++rep) {
        std::vector<uint64_t> r(n);
        for (auto& x : r) x = rng() % (span / 256);
        if (sorted == 1) std::sort(r.begin(), r.end());
        if (sorted == 2) {  // sorted within warps of 32 only
          for (int64_t i = 0; i < n; i += 32) std::sort(r.begin() + i, r.begin() + std::min<int64_t>(n, i + 32));
        }
        cudaMemcpy(drows, r.data(), 8 * n, cudaMemcpyHostToDevice);
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        cudaEventRecord(a);
        list_probe<<<(n + 127) / 128, 128>>>((const float*)d, drows, n, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        best = std::min(best, (double)ms);
      }
      printf("\"n%ld_%s_us\": %.1f, ", (long)n, sorted == 0 ? "random" : (sorted == 1 ? "sorted" : "warpsorted"),
             best * 1e3);
    }
  }
  printf("\"done\": 1}\n");
  return 0;
}
