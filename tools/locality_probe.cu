// tools/locality_probe.cu — what limits random-row zero-copy reads at large spans?
// Random 256 B rows from a mapped pinned host buffer, where each group of k consecutive
// lanes draws rows from the SAME page of 2^shift bytes (k = 1: uniform).  If the rows/s
// rate scales with k for some page size, one translation per such page is the limiter.
#include <cuda_runtime.h>

#include <cstdio>

#include "kernels.cuh"

template <int D>
__global__ void __launch_bounds__(128) grouped_probe(const float* host, uint64_t pages, uint64_t rows_per_page,
                                                     int64_t rows, int k, uint64_t seed, float* sink) {
  const int lane = threadIdx.x & 31;
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g - lane >= rows) return;
  const bool active = g < rows;
  const uint64_t page = fl::splitmix64(seed ^ (uint64_t)(g / k)) % pages;
  const uint64_t r = page * rows_per_page + fl::splitmix64(seed + (uint64_t)g) % rows_per_page;
  const float* src = active ? host + r * (uint64_t)D : nullptr;
  float* dst = active ? sink + (size_t)(g & 4095) * D : nullptr;
  fl::gather_rows<D>(src, dst, lane);
}

int main() {
  cudaSetDevice(0);
  float* sink;
  cudaMalloc(&sink, 4096 * 512);
  printf("{");
  for (size_t span : {1ull << 30, 8ull << 30}) {
    void* h;
    if (cudaHostAlloc(&h, span, cudaHostAllocMapped) != cudaSuccess) continue;
    cudaMemset(h, 1, span);
    void* d;
    cudaHostGetDevicePointer(&d, h, 0);
    for (int shift : {21, 16, 12}) {
      const uint64_t rpp = (1ull << shift) / 256, pages = span >> shift;
      for (int k : {1, 4, 16}) {
        const int64_t rows = 1 << 20;
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        grouped_probe<64><<<(rows + 127) / 128, 128>>>((const float*)d, pages, rpp, rows, k, 3, sink);
        cudaEventRecord(a);
        grouped_probe<64><<<(rows + 127) / 128, 128>>>((const float*)d, pages, rpp, rows, k, 5, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("\"span%zuG_page2^%d_k%d_Mrows\": %.1f, ", span >> 30, shift, k, rows / (ms * 1e3));
      }
    }
    cudaFreeHost(h);
    fflush(stdout);
  }
  printf("\"done\": 1}\n");
  return 0;
}
