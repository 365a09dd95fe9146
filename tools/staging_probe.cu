// tools/staging_probe.cu — how fast does a KM-shaped read of a small contiguous pinned
// staging buffer go with each load flavour?  W warps each read B bytes (16 B per lane
// per load, 16 loads in flight per lane) of a cudaHostAlloc'd buffer into shared memory.
// Optionally NT host threads rewrite the buffer concurrently (the host-assisted pattern).
#include <cuda_runtime.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <thread>
#include <vector>

template <int MODE>
__device__ __forceinline__ float4 ld(const float* p) {
  float4 v;
  if (MODE == 0) asm volatile("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  if (MODE == 1) asm volatile("ld.global.cv.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p) : "memory");
  if (MODE == 2) asm volatile("ld.relaxed.sys.global.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p) : "memory");
  if (MODE == 3) asm volatile("ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p) : "memory");
  if (MODE == 4) asm volatile("ld.volatile.global.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p) : "memory");
  return v;
}

template <int MODE>
__global__ void __launch_bounds__(128) rd(const float* src, size_t per_warp_f4, float* sink) {
  __shared__ float4 sm[4][512];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const size_t gw = (size_t)blockIdx.x * 4 + w;
  const float* base = src + gw * per_warp_f4 * 4;
  for (size_t q0 = 0; q0 < per_warp_f4 / 32; q0 += 16) {
    float4 v[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = ld<MODE>(base + 4 * ((q0 + i) * 32 + lane));
#pragma unroll
    for (int i = 0; i < 16; ++i) sm[w][((q0 + i) * 32 + lane) & 511] = v[i];
  }
  __syncwarp();
  if (sm[w][lane].x == 12345.f) sink[0] = 1.f;
}

int main() {
  cudaSetDevice(0);
  const size_t bytes = 64ull << 20;
  void* h;
  cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable);
  memset(h, 0, bytes);
  void* d;
  cudaHostGetDevicePointer(&d, h, 0);
  float* sink;
  cudaMalloc(&sink, 1024);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  std::atomic<bool> stop{false};
  printf("{");
  for (int writers : {0, 12}) {
    stop = false;
    std::vector<std::thread> th;
    for (int t = 0; t < writers; ++t)
      th.emplace_back([&, t]() {  // rewrite the second half of the buffer, like staging of later blocks
        char* p = (char*)h + bytes / 2 + (size_t)t * (bytes / 2 / 16);
        while (!stop) memset(p, t, bytes / 2 / 16);
      });
    for (int warps : {128, 512}) {
      for (size_t kb : {16, 64}) {
        const size_t per_warp_f4 = kb * 1024 / 16;
        if (warps * kb * 1024 > bytes / 2) continue;
        const unsigned blocks = warps / 4;
        for (int mode = 0; mode < 5; ++mode) {
          float best = 1e30f;
          for (int rep = 0; rep < 5; ++rep) {
            cudaEventRecord(e0);
            if (mode == 0) rd<0><<<blocks, 128>>>((const float*)d, per_warp_f4, sink);
            if (mode == 1) rd<1><<<blocks, 128>>>((const float*)d, per_warp_f4, sink);
            if (mode == 2) rd<2><<<blocks, 128>>>((const float*)d, per_warp_f4, sink);
            if (mode == 3) rd<3><<<blocks, 128>>>((const float*)d, per_warp_f4, sink);
            if (mode == 4) rd<4><<<blocks, 128>>>((const float*)d, per_warp_f4, sink);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            best = ms < best ? ms : best;
          }
          const char* nm[] = {"nc", "cv", "relaxed_sys", "cg", "volatile"};
          printf("%s\"w%d_%s_%dwarps_%zuKB\": {\"us\": %.1f, \"gbs\": %.1f}", (writers || warps != 128 || kb != 16 || mode) ? ", " : "",
                 writers, nm[mode], warps, kb, best * 1e3, warps * kb * 1024 / (best * 1e-3) / 1e9);
          fflush(stdout);
        }
      }
    }
    stop = true;
    for (auto& t : th) t.join();
  }
  printf("}\n");
  return 0;
}
