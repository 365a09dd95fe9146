// tools/vmm_host_probe.cu — does the host-tier allocation method change the random-row
// zero-copy read rate?  Compares cudaHostAlloc (mapped pinned) with CUDA VMM host
// allocations (cuMemCreate, location HOST_NUMA, large granularity) over growing spans.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include
//        -I paper_conf_eurosys_xiellwgrs22_b200/csrc tools/vmm_host_probe.cu -lcuda -o tools/vmm_host_probe
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#include "kernels.cuh"

#define CK(x)                                                                 \
  do {                                                                        \
    CUresult r_ = (x);                                                        \
    if (r_ != CUDA_SUCCESS) {                                                 \
      const char* s_;                                                         \
      cuGetErrorString(r_, &s_);                                              \
      printf("{\"error\": \"%s -> %s\"}\n", #x, s_);                          \
      return 1;                                                               \
    }                                                                         \
  } while (0)

static double probe(const float* dev, size_t bytes, int row, long rows, float* sink) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const uint64_t span = bytes / row;
  const unsigned blocks = (unsigned)((rows + 127) / 128);
  auto go = [&](uint64_t seed) {
    if (row == 128) fl::probe_host_kernel<32><<<blocks, 128>>>(dev, span, rows, seed, sink);
    else if (row == 256) fl::probe_host_kernel<64><<<blocks, 128>>>(dev, span, rows, seed, sink);
    else fl::probe_host_kernel<128><<<blocks, 128>>>(dev, span, rows, seed, sink);
  };
  go(99);
  cudaEventRecord(a);
  go(7);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  return rows * (double)row / (ms * 1e-3) / 1e9;
}

int main(int argc, char** argv) {
  cudaSetDevice(0);
  cudaFree(0);
  float* sink;
  cudaMalloc(&sink, 4096 * 512);
  std::vector<size_t> spans = {1ull << 30, 4ull << 30, 8ull << 30, 32ull << 30};
  printf("{");
  for (size_t span : spans) {
    // (1) cudaHostAlloc mapped
    void* h = nullptr;
    if (cudaHostAlloc(&h, span, cudaHostAllocMapped | cudaHostAllocPortable) == cudaSuccess) {
      cudaMemset(h, 1, span);
      cudaDeviceSynchronize();
      void* d;
      cudaHostGetDevicePointer(&d, h, 0);
      for (int row : {128, 256, 512})
        printf("\"hostalloc_%zuG_%dB\": %.2f, ", span >> 30, row, probe((const float*)d, span, row, 1 << 21, sink));
      cudaFreeHost(h);
    }
    // (2) VMM host allocation
    CUmemAllocationProp prop = {};
    prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    prop.location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA;
    prop.location.id = 0;
    size_t gran = 0;
    CK(cuMemGetAllocationGranularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED));
    size_t sz = (span + gran - 1) / gran * gran;
    CUmemGenericAllocationHandle hd;
    CK(cuMemCreate(&hd, sz, &prop, 0));
    CUdeviceptr va;
    CK(cuMemAddressReserve(&va, sz, 1ull << 30, 0, 0));
    CK(cuMemMap(va, sz, 0, hd, 0));
    CUmemAccessDesc acc[2] = {};
    acc[0].location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    acc[0].location.id = 0;
    acc[0].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    acc[1].location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA;
    acc[1].location.id = 0;
    acc[1].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CUresult ra = cuMemSetAccess(va, sz, acc, 2);
    if (ra != CUDA_SUCCESS) CK(cuMemSetAccess(va, sz, acc, 1));
    printf("\"vmm_gran_MiB\": %zu, \"vmm_host_access\": %d, ", gran >> 20, ra == CUDA_SUCCESS);
    cudaMemset((void*)va, 1, sz);
    cudaDeviceSynchronize();
    if (ra == CUDA_SUCCESS) ((volatile float*)va)[12345] = 2.0f;  // host touch works?
    for (int row : {128, 256, 512})
      printf("\"vmm_%zuG_%dB\": %.2f, ", span >> 30, row, probe((const float*)va, span, row, 1 << 21, sink));
    CK(cuMemUnmap(va, sz));
    CK(cuMemAddressFree(va, sz));
    CK(cuMemRelease(hd));
    // (3) device memory, for scale
    if (span <= (32ull << 30)) {
      void* dm;
      if (cudaMalloc(&dm, span) == cudaSuccess) {
        cudaMemset(dm, 1, span);
        printf("\"hbm_%zuG_256B\": %.2f, ", span >> 30, probe((const float*)dm, span, 256, 1 << 23, sink));
        cudaFree(dm);
      }
    }
    fflush(stdout);
  }
  printf("\"done\": 1}\n");
  return 0;
}
