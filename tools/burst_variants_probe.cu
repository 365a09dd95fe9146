// tools/burst_variants_probe.cu — how should the miss kernel issue one batch's host-row
// reads?  One burst = R random 256 B rows of an 8 GiB mapped pinned buffer (uniform over
// the span, like cfg2's unique misses), every row copied to HBM.  Variants:
//   ldg16  one warp per 32 rows, 16 lanes x 16 B per row, 16 rows in flight per warp (the
//          current gather_rows<64>: two rounds per warp)
//   ldg32  one warp per 32 rows, all 32 rows' loads in flight before any store
//   cpa    one warp per 32 rows, cp.async 16 B (LDGSTS) into shared memory, all in flight
//   bulk   one warp per 32 rows, cp.async.bulk (TMA engine) 256 B per row into shared
//          memory, completion on an mbarrier
//   km8    a fixed grid of 592 warps (KM's), 8 rows per warp per round, rounds in sequence
//          (the current miss kernel's issue pattern)
//   km8s   same with the rows of a round issued in address order (sorted burst)
// Reports µs per burst (mean of 8 bursts with fresh seeds).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "kernels.cuh"

using namespace fl;

__device__ __forceinline__ uint64_t row_of(uint64_t seed, uint64_t g, uint64_t rows) {
  return splitmix64(seed + g) % rows;
}

template <int MODE>
__global__ void __launch_bounds__(128) burst(const float* host, uint64_t all_rows, int64_t R, uint64_t seed,
                                             float* sink, const uint64_t* order) {
  __shared__ __align__(128) float4 sm[4][32][16];
  __shared__ __align__(8) unsigned long long mbar[4];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t w = (int64_t)blockIdx.x * 4 + wib;
  const int64_t g = w * 32 + lane;
  if (w * 32 >= R) return;
  const bool active = g < R;
  const uint64_t r = order ? order[g < R ? g : 0] : row_of(seed, (uint64_t)g, all_rows);
  const float* src = active ? host + r * 64ull : nullptr;
  float* dst = active ? sink + (size_t)(g & 16383) * 64 : nullptr;
  if constexpr (MODE == 0) {
    gather_rows<64>(src, dst, lane);
  } else if constexpr (MODE == 1) {
    float4 v[16];
    const int sub = lane & 15, rs = lane >> 4;
#pragma unroll
    for (int p = 0; p < 16; ++p) {
      const float* s = (const float*)__shfl_sync(kFull, (unsigned long long)src, 2 * p + rs);
      v[p] = s ? ld_nc_v4(s + 4 * sub) : make_float4(0, 0, 0, 0);
    }
#pragma unroll
    for (int p = 0; p < 16; ++p) {
      float* o = (float*)__shfl_sync(kFull, (unsigned long long)dst, 2 * p + rs);
      if (o) st_v4(o + 4 * sub, v[p]);
    }
  } else if constexpr (MODE == 2) {
    const int sub = lane & 15, rs = lane >> 4;
#pragma unroll
    for (int p = 0; p < 16; ++p) {
      const float* s = (const float*)__shfl_sync(kFull, (unsigned long long)src, 2 * p + rs);
      if (s) {
        const unsigned sa = (unsigned)__cvta_generic_to_shared(&sm[wib][2 * p + rs][sub]);
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sa), "l"(s + 4 * sub) : "memory");
      }
    }
    asm volatile("cp.async.commit_group;\n\tcp.async.wait_all;" ::: "memory");
    __syncwarp();
#pragma unroll
    for (int p = 0; p < 16; ++p) {
      float* o = (float*)__shfl_sync(kFull, (unsigned long long)dst, 2 * p + rs);
      if (o) st_v4(o + 4 * sub, sm[wib][2 * p + rs][sub]);
    }
  } else if constexpr (MODE == 3) {
    const unsigned mb = (unsigned)__cvta_generic_to_shared(&mbar[wib]);
    const unsigned nrows = __popc(__ballot_sync(kFull, active));
    if (lane == 0) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb) : "memory");
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    if (lane == 0)
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(nrows * 256u) : "memory");
    __syncwarp();
    if (active) {
      const unsigned sa = (unsigned)__cvta_generic_to_shared(&sm[wib][lane][0]);
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 256, [%2];" ::"r"(sa),
                   "l"(src), "r"(mb)
                   : "memory");
    }
    asm volatile(
        "{\n\t.reg .pred p;\n\tLAB_WAIT:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n\t"
        "@!p bra LAB_WAIT;\n\t}" ::"r"(mb)
        : "memory");
    const int sub = lane & 15, rs = lane >> 4;
#pragma unroll
    for (int p = 0; p < 16; ++p) {
      float* o = (float*)__shfl_sync(kFull, (unsigned long long)dst, 2 * p + rs);
      if (o) st_v4(o + 4 * sub, sm[wib][2 * p + rs][sub]);
    }
  }
}

// KM's pattern: nw warps, rounds of 8 rows per warp (lanes 0..7 hold the rows)
__global__ void __launch_bounds__(128) burst_km(const float* host, uint64_t all_rows, int64_t R, uint64_t seed,
                                                float* sink, const uint64_t* order) {
  const int lane = threadIdx.x & 31;
  const uint32_t gw = (threadIdx.x >> 5) * gridDim.x + blockIdx.x;
  const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
  for (int64_t base = (int64_t)gw * 8; base < R; base += (int64_t)nw * 8) {
    const int64_t g = base + lane;
    const bool has = lane < 8 && g < R;
    const uint64_t r = has ? (order ? order[g] : row_of(seed, (uint64_t)g, all_rows)) : 0;
    RowBuf<64, 8> rb;
    rb.load(has ? host + r * 64ull : nullptr, lane);
    rb.store(has ? sink + (size_t)(g & 16383) * 64 : nullptr, lane);
  }
}

static uint64_t h_splitmix(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

#include <sys/mman.h>

int main(int argc, char** argv) {
  // argv[1]: host allocation: "hostalloc" (cudaHostAlloc), "malloc" (malloc + cudaHostRegister,
  // 4 KiB pages), "thp" (mmap + MADV_HUGEPAGE + cudaHostRegister), "hugetlb" (MAP_HUGETLB 2 MiB)
  const char* mode = argc > 1 ? argv[1] : "hostalloc";
  cudaSetDevice(0);
  float* sink;
  cudaMalloc(&sink, 16384 * 256);
  const size_t span = 8ull << 30;
  void* h = nullptr;
  if (!strcmp(mode, "hostalloc")) {
    if (cudaHostAlloc(&h, span, cudaHostAllocMapped) != cudaSuccess) return 1;
  } else if (!strcmp(mode, "malloc")) {
    h = aligned_alloc(4096, span);
  } else {
    const int fl = MAP_PRIVATE | MAP_ANONYMOUS | (!strcmp(mode, "hugetlb") ? MAP_HUGETLB : 0);
    h = mmap(nullptr, span, PROT_READ | PROT_WRITE, fl, -1, 0);
    if (h == MAP_FAILED) { fprintf(stderr, "mmap failed\n"); return 1; }
    if (!strcmp(mode, "thp")) madvise(h, span, MADV_HUGEPAGE);
  }
  memset(h, 1, span);
  if (strcmp(mode, "hostalloc") && cudaHostRegister(h, span, cudaHostRegisterMapped) != cudaSuccess) {
    fprintf(stderr, "register failed\n");
    return 1;
  }
  float* d;
  cudaHostGetDevicePointer((void**)&d, h, 0);
  const uint64_t all_rows = span / 256;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  uint64_t* d_order;
  cudaMalloc(&d_order, 65536 * 8);
  printf("{\"alloc\": \"%s\", ", mode);
  for (int64_t R : {2048, 8192, 32768}) {
    auto timeit = [&](auto&& body) {
      body(0xABCDEF1234567ull);
      cudaDeviceSynchronize();
      float tot = 0;
      for (int it = 0; it < 8; ++it) {
        cudaEventRecord(a);
        body((uint64_t)(it + 1) * 0x9E3779B97F4A7C15ull);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        tot += ms;
      }
      return tot / 8 * 1000.0f;
    };
    const unsigned blocks = (unsigned)((R + 127) / 128);
    const float t0 = timeit([&](uint64_t s) { burst<0><<<blocks, 128>>>(d, all_rows, R, s, sink, nullptr); });
    const float t1 = timeit([&](uint64_t s) { burst<1><<<blocks, 128>>>(d, all_rows, R, s, sink, nullptr); });
    const float t2 = timeit([&](uint64_t s) { burst<2><<<blocks, 128>>>(d, all_rows, R, s, sink, nullptr); });
    const float t3 = timeit([&](uint64_t s) { burst<3><<<blocks, 128>>>(d, all_rows, R, s, sink, nullptr); });
    const float t4 = timeit([&](uint64_t s) { burst_km<<<592, 128>>>(d, all_rows, R, s, sink, nullptr); });
    // sorted bursts: host generates the same rows and sorts them (address order)
    std::vector<std::vector<uint64_t>> ord(9);
    for (int it = 0; it < 9; ++it) {
      const uint64_t sd = it == 0 ? 0xABCDEF1234567ull : (uint64_t)it * 0x9E3779B97F4A7C15ull;
      ord[it].resize(R);
      for (int64_t g = 0; g < R; ++g) ord[it][g] = h_splitmix(sd + g) % all_rows;
      std::sort(ord[it].begin(), ord[it].end());
    }
    int k = 0;
    const float t5 = timeit([&](uint64_t) {
      cudaMemcpy(d_order, ord[k++ % 9].data(), R * 8, cudaMemcpyHostToDevice);
      cudaEventRecord(a);
      burst_km<<<592, 128>>>(d, all_rows, R, 0, sink, d_order);
    });
    k = 0;
    const float t6 = timeit([&](uint64_t) {
      cudaMemcpy(d_order, ord[k++ % 9].data(), R * 8, cudaMemcpyHostToDevice);
      cudaEventRecord(a);
      burst<1><<<blocks, 128>>>(d, all_rows, R, 0, sink, d_order);
    });
    printf("\"R%lld\": {\"ldg16\": %.1f, \"ldg32\": %.1f, \"cpa\": %.1f, \"bulk\": %.1f, \"km8\": %.1f, "
           "\"km8_sorted\": %.1f, \"ldg32_sorted\": %.1f}, ",
           (long long)R, t0, t1, t2, t3, t4, t5, t6);
    fflush(stdout);
  }
  printf("\"done\": 1}\n");
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) fprintf(stderr, "%s\n", cudaGetErrorString(e));
  return 0;
}
