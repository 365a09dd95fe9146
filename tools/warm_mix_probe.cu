// tools/warm_mix_probe.cu — can a compact "warm" host region dodge the translation limit
// of scattered zero-copy reads while cold reads over a large span are in flight?
//
// One burst = R rows of 256 B (one row per lane, 16 B vector loads): a share f of them
// random inside the first W bytes of an 8 GiB mapped pinned buffer (the warm region),
// the rest random over the whole buffer (cold).  Reports µs per burst (mean of 8
// bursts with fresh seeds) for f in {0, .25, .5, .75, 1} and W in {256 MiB, 1 GiB}, with
// the warm and cold rows interleaved in one kernel or issued as two kernels on two
// streams.  Also: random 256 B row writes (GPU -> host) into the warm region, alone and
// concurrent with a cold read burst (the cost of writing evicted rows back to the host).
#include <cuda_runtime.h>

#include <cstdio>
#include <vector>

#include "kernels.cuh"

__global__ void __launch_bounds__(128) mix_read(const float* host, uint64_t warm_rows, uint64_t all_rows, int64_t rows,
                                                uint32_t warm_q16, uint64_t seed, float* sink) {
  const int lane = threadIdx.x & 31;
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g - lane >= rows) return;
  const bool active = g < rows;
  const uint64_t h = fl::splitmix64(seed + (uint64_t)g);
  const bool warm = (uint32_t)(h & 0xFFFF) < warm_q16;
  const uint64_t r = (h >> 16) % (warm ? warm_rows : all_rows);
  const float* src = active ? host + r * 64ull : nullptr;
  float* dst = active ? sink + (size_t)(g & 8191) * 64 : nullptr;
  fl::gather_rows<64>(src, dst, lane);
}

__global__ void __launch_bounds__(128) warm_write(float* host, uint64_t warm_rows, int64_t rows, uint64_t seed,
                                                  const float* src) {
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & 31;
  if (g - lane >= rows) return;
  const bool active = g < rows;
  const uint64_t r = fl::splitmix64(seed + (uint64_t)g) % warm_rows;
  // row r <- src row (g & 8191): 16 lanes x 16 B per row, lanes take the warp's rows in turn
  for (int k = 0; k < 32; ++k) {
    const int64_t gk = __shfl_sync(fl::kFull, g, k);
    const uint64_t rk = __shfl_sync(fl::kFull, r, k);
    const bool ak = __shfl_sync(fl::kFull, active, k);
    if (!ak || lane >= 16) continue;
    const float4 v = *reinterpret_cast<const float4*>(src + (size_t)(gk & 8191) * 64 + 4 * lane);
    *reinterpret_cast<float4*>(host + rk * 64ull + 4 * lane) = v;
  }
}

int main() {
  cudaSetDevice(0);
  float* sink;
  cudaMalloc(&sink, 8192 * 256);
  cudaMemset(sink, 0, 8192 * 256);
  const size_t span = 8ull << 30;
  void* h;
  if (cudaHostAlloc(&h, span, cudaHostAllocMapped) != cudaSuccess) return 1;
  cudaMemset(h, 1, span);
  float* d;
  cudaHostGetDevicePointer((void**)&d, h, 0);
  cudaStream_t s1, s2;
  cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
  cudaEvent_t a, b, j;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventCreate(&j);
  const uint64_t all_rows = span / 256;
  auto timeit = [&](auto&& body) {
    body(0xABCDEF1234567ull);  // warm-up
    cudaDeviceSynchronize();
    float tot = 0;
    for (int it = 0; it < 8; ++it) {
      cudaEventRecord(a, s1);
      cudaStreamWaitEvent(s2, a, 0);
      body((uint64_t)(it + 1) * 0x9E3779B97F4A7C15ull);
      cudaEventRecord(j, s2);
      cudaStreamWaitEvent(s1, j, 0);
      cudaEventRecord(b, s1);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      tot += ms;
    }
    return tot / 8 * 1000.0f;
  };
  printf("{");
  for (int64_t R : {8192, 32768}) {
    for (uint64_t W : {256ull << 20, 1ull << 30}) {
      const uint64_t warm_rows = W / 256;
      for (double f : {0.0, 0.25, 0.5, 0.75, 1.0}) {
        const uint32_t q = (uint32_t)(f * 65536.0);
        const float us1 = timeit([&](uint64_t sd) {
          mix_read<<<(R + 127) / 128, 128, 0, s1>>>(d, warm_rows, all_rows, R, q, sd, sink);
        });
        // two kernels on two streams: warm rows and cold rows concurrently
        const int64_t Rw = (int64_t)(R * f), Rc = R - Rw;
        const float us2 = timeit([&](uint64_t sd) {
          if (Rw) mix_read<<<(Rw + 127) / 128, 128, 0, s1>>>(d, warm_rows, all_rows, Rw, 65536u, sd, sink);
          if (Rc) mix_read<<<(Rc + 127) / 128, 128, 0, s2>>>(d, warm_rows, all_rows, Rc, 0u, sd ^ 99, sink);
        });
        // two kernels in sequence: warm rows first, then cold
        const float us3 = timeit([&](uint64_t sd) {
          if (Rw) mix_read<<<(Rw + 127) / 128, 128, 0, s1>>>(d, warm_rows, all_rows, Rw, 65536u, sd, sink);
          if (Rc) mix_read<<<(Rc + 127) / 128, 128, 0, s1>>>(d, warm_rows, all_rows, Rc, 0u, sd ^ 99, sink);
        });
        printf("\"R%lld_W%lluM_f%.2f_us\": [%.1f, %.1f, %.1f], ", (long long)R, (unsigned long long)(W >> 20), f, us1,
               us2, us3);
        fflush(stdout);
      }
      // write-back: R random row writes into the warm region, alone / concurrent with R cold reads
      const float w1 = timeit([&](uint64_t sd) {
        warm_write<<<(R + 127) / 128, 128, 0, s2>>>(d, warm_rows, R, sd, sink);
      });
      const float w2 = timeit([&](uint64_t sd) {
        mix_read<<<(R + 127) / 128, 128, 0, s1>>>(d, warm_rows, all_rows, R, 0u, sd, sink);
        warm_write<<<(R + 127) / 128, 128, 0, s2>>>(d, warm_rows, R, sd ^ 5, sink);
      });
      const float w3 = timeit([&](uint64_t sd) {
        mix_read<<<(R + 127) / 128, 128, 0, s1>>>(d, warm_rows, all_rows, R, 0u, sd, sink);
      });
      printf("\"R%lld_W%lluM_write_alone_us\": %.1f, \"R%lld_W%lluM_write_with_cold_read_us\": %.1f, "
             "\"R%lld_cold_read_alone_us\": %.1f, ",
             (long long)R, (unsigned long long)(W >> 20), w1, (long long)R, (unsigned long long)(W >> 20), w2,
             (long long)R, w3);
      fflush(stdout);
    }
  }
  printf("\"done\": 1}\n");
  cudaFreeHost(h);
  return 0;
}
