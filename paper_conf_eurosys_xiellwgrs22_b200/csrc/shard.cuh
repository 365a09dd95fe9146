// shard.cuh — key-sharded multi-GPU mode: the device side.
//
// Each rank caches the keys it OWNS, owner(fk) = (fmix32(fk ^ seed') * G) >> 32, so the
// aggregate cache capacity is G x the per-GPU budget (the paper leaves multi-GPU caching
// to future work).  Per batch, on every rank:
//   KR  route: dedup the batch's valid flat keys (epoch-tagged scratch) and group the
//       unique keys by owner;                               (device)
//   KPK pack: owner-grouped keys -> one contiguous send buffer + per-owner counts;
//       all-to-all of counts, of keys (NCCL, NVLink)        (host plumbing: torch.distributed)
//   ... the owner answers its received keys with the ordinary KQ/KM/KD path in flat-key
//       mode (fleche_query_keys), all-to-all of rows (+ per-key hit flags) back ...
//   KRS restore: every lookup copies its key's row from the received rows.
#pragma once
#include <cstdint>

#include "kernels.cuh"

namespace fl {

constexpr int kMaxWorld = 64;

struct RouteDev {
  unsigned long long* scratch;  // [mask+1] (route epoch << 32 | fk)
  unsigned long long* slotval;  // [mask+1] (owner << 32 | index in the owner's group)
  uint32_t* inv;                // [max_lookups] scratch slot of each lookup (kEmpty = invalid ID)
  uint32_t* region;             // [world][cap] unique keys grouped by owner
  uint32_t* cnt;                // [kMaxWorld] unique keys per owner (this batch)
  int64_t* prefix;              // [kMaxWorld + 1] exclusive prefix of cnt (saved by KPK)
  uint32_t* done;               // KPK CTA arrival counter
  unsigned long long* stats;    // [4]: lookups, per-lookup hits, invalid, unique routed keys
  uint32_t mask, cap;
  int32_t world;
  uint32_t owner_seed;
};

// Fused key-sharded exchange (fleche_restore_p2p): each owner's answer rows and hit
// flags are read in place through peer pointers (CUDA IPC over NVLink); off[o] = where
// this rank's keys start in owner o's received order.
struct PeerArgs {
  const float* rows[kMaxWorld];
  const uint8_t* flags[kMaxWorld];
  int64_t off[kMaxWorld];
  int32_t p2p;
  int32_t me;             // sync-free variant: this rank, and
  const int64_t* dcnt;    // the [world][world] routed-count matrix in device memory (off[] unused)
};

// Fused exchange, key side (fleche_route_p2p): dst[o] = this rank's slot in owner o's
// receive buffer (a peer pointer through CUDA IPC; own buffer for o == rank).
struct PeerKeys {
  uint32_t* dst[kMaxWorld];
  int32_t p2p;
  int32_t pad;
};

template <int MAXT>
struct RArgs {
  const int64_t* ids[MAXT];
  int64_t scan[MAXT + 1];
  int64_t out_off[MAXT];
  int32_t n;
  uint32_t repoch;
};

__device__ __forceinline__ uint32_t owner_of(uint32_t fk, uint32_t seed, int world) {
  return __umulhi(fmix32(fk ^ seed ^ 0x85EBCA77u), (uint32_t)world);
}

template <int MAXT>
__device__ __forceinline__ int find_table(const int64_t* s_scan, int n, int64_t g) {
  int lo = 0, hi = n;
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (s_scan[mid] <= g) lo = mid; else hi = mid;
  }
  return lo;
}

template <int MAXT>
__global__ void __launch_bounds__(128) kr_kernel(const __grid_constant__ RArgs<MAXT> ra, const __grid_constant__ RouteDev rd,
                                                 const TableInfo* __restrict__ tables) {
  __shared__ int64_t s_scan[MAXT + 1];
  __shared__ unsigned long long s_ctr[4];
  for (int i = threadIdx.x; i <= ra.n; i += blockDim.x) s_scan[i] = ra.scan[i];
  if (threadIdx.x < 4) s_ctr[threadIdx.x] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t N = s_scan[ra.n];
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g - lane < N) {
    const bool active = g < N;
    int t = 0;
    int64_t id = -1;
    if (active) {
      t = find_table<MAXT>(s_scan, ra.n, g);
      id = ra.ids[t][g - s_scan[t]];
    }
    const TableInfo* ti = tables + t;
    const bool valid = active && id >= 0 && id < ti->card;
    const uint32_t fk = valid ? ti->base + (uint32_t)id : kEmpty;
    int kind = 0;
    uint32_t scr = kEmpty;
    if (valid) {
      const unsigned long long tag = ((unsigned long long)ra.repoch << 32) | fk;
      uint32_t h = scr_hash(fk ^ 0x27D4EB2Fu) & rd.mask;
      unsigned long long cur = ld_cg_u64(rd.scratch + h);
      while (true) {
        if (cur == tag) { kind = 2; break; }
        if ((uint32_t)(cur >> 32) != ra.repoch) {
          const unsigned long long prev = atomicCAS(rd.scratch + h, cur, tag);
          if (prev == cur) { kind = 1; break; }
          cur = prev;
          continue;
        }
        h = (h + 1) & rd.mask;
        cur = ld_cg_u64(rd.scratch + h);
      }
      scr = h;
    }
    const unsigned own_m = __ballot_sync(kFull, kind == 1);
    if (own_m) {  // append to the owner's group, aggregated per owner within the warp
      const uint32_t o = kind == 1 ? owner_of(fk, rd.owner_seed, rd.world) : 0u;
      const unsigned grp = __match_any_sync(kFull, kind == 1 ? (int)o : 1024 + lane);
      const int leader = __ffs(grp) - 1;
      uint32_t b = 0;
      if (kind == 1 && lane == leader) b = atomicAdd(rd.cnt + o, (uint32_t)__popc(grp));
      b = __shfl_sync(kFull, b, leader);
      if (kind == 1) {
        const uint32_t i = b + __popc(grp & ((1u << lane) - 1u));
        rd.region[(size_t)o * rd.cap + i] = fk;
        rd.slotval[scr] = ((unsigned long long)o << 32) | i;
      }
    }
    if (active) rd.inv[g] = scr;
    const unsigned am = __ballot_sync(kFull, active), im = __ballot_sync(kFull, active && !valid);
    if (lane == 0) {
      atomicAdd(&s_ctr[0], (unsigned long long)__popc(am));
      if (im) atomicAdd(&s_ctr[2], (unsigned long long)__popc(im));
      if (own_m) atomicAdd(&s_ctr[3], (unsigned long long)__popc(own_m));
    }
  }
  __syncthreads();
  if (threadIdx.x < 4 && s_ctr[threadIdx.x]) atomicAdd(rd.stats + threadIdx.x, s_ctr[threadIdx.x]);
}

// KPK: owner groups -> contiguous send buffer; counts out; the last CTA clears the
// per-owner counters for the next batch.
template <int = 0>
__global__ void __launch_bounds__(256) kpk_kernel(const __grid_constant__ RouteDev rd, uint32_t* __restrict__ send_keys,
                                                  int64_t* __restrict__ send_counts, const __grid_constant__ PeerKeys pk) {
  __shared__ int64_t s_pre[kMaxWorld + 1];
  __shared__ uint32_t s_cnt[kMaxWorld];
  if (threadIdx.x == 0) {
    int64_t acc = 0;
    for (int o = 0; o < rd.world; ++o) {
      s_cnt[o] = *(volatile uint32_t*)(rd.cnt + o);
      s_pre[o] = acc;
      acc += s_cnt[o];
    }
    s_pre[rd.world] = acc;
  }
  __syncthreads();
  const int64_t total = s_pre[rd.world];
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (int64_t)gridDim.x * blockDim.x) {
    int o = 0;
    while (s_pre[o + 1] <= k) ++o;
    const uint32_t key = rd.region[(size_t)o * rd.cap + (k - s_pre[o])];
    if (pk.p2p) pk.dst[o][k - s_pre[o]] = key;  // fused exchange: straight into owner o's slot (peer HBM)
    else send_keys[k] = key;
  }
  if (blockIdx.x == 0 && threadIdx.x < rd.world) {
    send_counts[threadIdx.x] = s_cnt[threadIdx.x];
    rd.prefix[threadIdx.x] = s_pre[threadIdx.x];
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(rd.done, 1u) == gridDim.x - 1) {
      for (int o = 0; o < rd.world; ++o) rd.cnt[o] = 0;
      *rd.done = 0;
      __threadfence();
    }
  }
}

// KRS: out row of every lookup = its key's row among the rows received back (owners
// return rows in the order the keys were sent); invalid IDs give a zero row.
template <int MAXT, int D>
__global__ void __launch_bounds__(128) krs_kernel(const __grid_constant__ RArgs<MAXT> ra, const __grid_constant__ RouteDev rd,
                                                  const float* __restrict__ rows, const uint8_t* __restrict__ flags,
                                                  float* __restrict__ out, const __grid_constant__ PeerArgs pa) {
  __shared__ int64_t s_scan[MAXT + 1];
  __shared__ int64_t s_off[kMaxWorld];
  __shared__ unsigned long long s_hits;
  for (int i = threadIdx.x; i <= ra.n; i += blockDim.x) s_scan[i] = ra.scan[i];
  if (threadIdx.x == 0) s_hits = 0;
  if (pa.p2p) {  // where this rank's keys start in each owner's received order
    for (int o = threadIdx.x; o < rd.world; o += blockDim.x) {
      int64_t acc = pa.off[o];
      if (pa.dcnt) {  // sync-free: sum of the counts owner o received from ranks < me
        acc = 0;
        for (int src = 0; src < pa.me; ++src) acc += pa.dcnt[(size_t)src * rd.world + o];
      }
      s_off[o] = acc;
    }
  }
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t N = s_scan[ra.n];
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g - lane < N) {
    const bool active = g < N;
    const float* src = nullptr;
    float* dst = nullptr;
    bool hit = false;
    if (active) {
      const int t = find_table<MAXT>(s_scan, ra.n, g);
      dst = out + ra.out_off[t] + (g - s_scan[t]) * D;
      const uint32_t scr = rd.inv[g];
      if (scr != kEmpty) {
        const unsigned long long v = rd.slotval[scr];
        if (!pa.p2p) {  // rows returned by the caller's all-to-all, in send order
          const int64_t pos = rd.prefix[v >> 32] + (int64_t)(v & 0xFFFFFFFFull);
          src = rows + pos * D;
          if (flags) hit = flags[pos] != 0;
        } else {  // fused exchange: read the owner's answer row where it lies (peer HBM over NVLink)
          const int o = (int)(v >> 32);
          const int64_t at = s_off[o] + (int64_t)(v & 0xFFFFFFFFull);
          src = pa.rows[o] + at * D;
          if (pa.flags[o]) hit = pa.flags[o][at] != 0;
        }
      }
    }
    gather_rows<D>(src, dst, lane);
    const unsigned hm = __ballot_sync(kFull, hit);
    if (lane == 0 && hm) atomicAdd(&s_hits, (unsigned long long)__popc(hm));
  }
  __syncthreads();
  if (threadIdx.x == 0 && s_hits) atomicAdd(rd.stats + 1, s_hits);
}

}  // namespace fl
