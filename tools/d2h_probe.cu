// D2H output-copy probe for fleche_query_host's e2e bound: one cfg2 output (54.5 MB fp32)
// HBM -> pinned host by (a) one cudaMemcpyAsync, (b) the same split over 2 / 4 streams
// (several copy engines), (c) SM stores into the mapped pinned buffer (zero-copy writes),
// 148 x k CTAs of 16 B stores.  Prints GB/s per variant (median of 20).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/d2h_probe tools/d2h_probe.cu
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdio>
#include <vector>

#define CK(x) do { cudaError_t err_ = (x); if (err_ != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(err_)); return 1; } } while (0)

__global__ void store_host(const float4* __restrict__ src, float4* dst, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    dst[i] = __ldcs(src + i);
}

int main() {
  const size_t bytes = 212992ull * 64 * 4;
  float *d, *h;
  CK(cudaMalloc(&d, bytes));
  CK(cudaMemset(d, 1, bytes));
  CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped));
  float* hd;
  CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
  cudaStream_t st[4];
  for (auto& s : st) CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t e0, e1, ej[4];
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  for (auto& e : ej) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  auto run = [&](const char* name, auto&& body) {
    std::vector<float> t;
    for (int r = 0; r < 23; ++r) {
      CK(cudaDeviceSynchronize());
      CK(cudaEventRecord(e0, st[0]));
      body();
      CK(cudaEventRecord(e1, st[0]));
      CK(cudaEventSynchronize(e1));
      float ms;
      CK(cudaEventElapsedTime(&ms, e0, e1));
      if (r >= 3) t.push_back(ms);
    }
    std::sort(t.begin(), t.end());
    printf("{\"variant\": \"%s\", \"ms\": %.4f, \"gbs\": %.2f}\n", name, t[t.size() / 2], bytes / (t[t.size() / 2] * 1e6));
    return 0;
  };
  auto split = [&](int k) {
    for (int i = 1; i < k; ++i) cudaStreamWaitEvent(st[i], e0, 0);
    const size_t chunk = (bytes / k + 255) & ~(size_t)255;
    for (int i = 0; i < k; ++i) {
      const size_t o = i * chunk, n = std::min(chunk, bytes - o);
      cudaMemcpyAsync((char*)h + o, (char*)d + o, n, cudaMemcpyDeviceToHost, st[i]);
    }
    for (int i = 1; i < k; ++i) { cudaEventRecord(ej[i], st[i]); cudaStreamWaitEvent(st[0], ej[i], 0); }
  };
  run("memcpy x1", [&] { split(1); });
  run("memcpy x2 streams", [&] { split(2); });
  run("memcpy x4 streams", [&] { split(4); });
  for (int k : {1, 2, 4, 8}) {
    char nm[64];
    snprintf(nm, sizeof nm, "sm stores 148x%d x256", k);
    run(nm, [&] { store_host<<<148 * k, 256, 0, st[0]>>>((const float4*)d, (float4*)hd, bytes / 16); });
  }
  printf("{\"check\": %s}\n", cudaGetLastError() == cudaSuccess ? "true" : "false");
  return 0;
}
