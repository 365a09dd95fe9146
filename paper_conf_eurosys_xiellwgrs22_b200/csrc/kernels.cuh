// kernels.cuh — device side of the B200 flat embedding cache (sm_100a).
//
// Two kernels per batch (the paper's "1 -> 2" after decoupling):
//
//   KQ  fused, self-identified query kernel: one lane per
//       lookup; each warp finds its table from the prefix offsets in shared memory,
//       re-encodes (table, id) to a flat key, probes its 32-way set with
//       a warp-cooperative ballot (index of P:L513-528), refreshes the hit way's
//       timestamp (approximate LRU), claims each unique missed key in an
//       epoch-tagged scratch table (dedup) and appends it to the miss
//       list, chains duplicate misses to their key, and copies hit rows from the HBM
//       slab into `out` with 16-byte vectors.  KQ never touches the host link.
//   KM  miss kernel (unified index + replacement, P:L855-860, P:L653-666,
//       P:L985-988): each warp takes up to 32 unique misses, issues all their
//       zero-copy host-row loads at once (pinned, mapped host tables), and while those
//       are in flight picks each miss's victim way (argmin (ts, key) over ways not
//       touched in this batch: epoch protection) and claims it with a CAS
//       on the way's timestamp; then writes the row to the owner's `out` position, to
//       every duplicate position (restore) and to the claimed slab slot,
//       and publishes the key.  The last CTA advances the device-resident epoch, so a
//       captured CUDA graph replays correctly.
//
// The hit copy (KQ, HBM-bound) is decoupled from the miss handling (KM, host-link
// bound): no lock is held across a copy and miss handling never waits on
// an index lock.
#pragma once
#include <cstdint>

namespace fl {

constexpr uint32_t kEmpty = 0xFFFFFFFFu;
constexpr unsigned kFull = 0xFFFFFFFFu;
constexpr int kStripes = 64;  // stats counters are striped to spread L2 atomics

enum Ctr : int {
  C_HITS = 0,
  C_MISSES,
  C_INVALID,
  C_UHITS,
  C_UMISS,
  C_INSERTED,
  C_EVICTED,
  C_BYPASSED,
  C_HOSTBYTES,
  C_DUPS,
  kNumCtr = 16
};

struct TableInfo {
  const float* host;  // device-visible address of E_t (mapped pinned host memory)
  int64_t card;       // c_t
  uint32_t base;      // first flat key of table t (size-aware coding)
  int32_t dim;        // d_t
};

struct MissRec {  // one unique missed key (its owner lookup)
  int64_t off;    // float offset of the owner's row in `out`
  uint32_t fk;    // flat key
  uint32_t scr;   // scratch slot of the key (head of its duplicate chain)
  int32_t t;      // table
  int32_t pad;
};

struct DupRec {  // a later occurrence of a missed key in the same batch
  int64_t off;   // float offset of the duplicate's row in `out`
  uint32_t next; // next duplicate + 1 (0 = end of chain)
  uint32_t pad;
};

struct Ctl {
  uint32_t epoch;  // current batch epoch (1-based); advanced by the last KM CTA
  uint32_t done;   // KM CTA arrival counter
  uint32_t err_invalid;
  uint32_t pad;
  uint32_t counts[2][4];  // [epoch & 1][0 = unique misses, 1 = duplicate misses]
  long long occ_rows;     // rows currently cached
};

struct Dev {
  uint32_t* keys;  // [sets][32] flat keys, kEmpty = free way
  uint32_t* ts;    // [sets][32] batch epoch of last touch (0 = never)
  float* slab;     // [sets*32][dim] rows; way w of set s at row s*32 + w
  unsigned long long* scratch;   // [scr_mask+1] (epoch << 32 | fk) dedup tags
  unsigned long long* dup_head;  // [scr_mask+1] (epoch << 32 | first duplicate + 1)
  MissRec* miss;                 // [max_lookups]
  DupRec* dup;                   // [max_lookups]
  Ctl* ctl;
  unsigned long long* stats;  // [kStripes][kNumCtr]
  const TableInfo* tables;    // [n]
  uint32_t sets, rows, scr_mask, hash_seed;
  int32_t dim, admit_all;
  uint64_t admit_thr, admit_seed;
  int32_t prefetch;  // KQ starts each unique miss's host-row transfer into L2
  int32_t km_m;      // unique misses per KM warp iteration (4, 8, 16, 32)
#ifdef FLECHE_EXPERIMENTS
  int32_t exp_mode;  // timing experiments only (libfleche_exp.so); breaks semantics
  int32_t exp_pad;
#endif
};

template <int MAXT>
struct QArgs {
  const int64_t* ids[MAXT];  // per-table device ID arrays
  int64_t scan[MAXT + 1];    // exclusive prefix of lengths
  int64_t out_off[MAXT];     // float offset of O_t in out
  float* out;
  int32_t n;
};

__device__ __forceinline__ uint32_t fmix32(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85EBCA6BU;
  h ^= h >> 13;
  h *= 0xC2B2AE35U;
  h ^= h >> 16;
  return h;
}
__device__ __forceinline__ uint32_t set_of(const Dev& dv, uint32_t fk) {
  return __umulhi(fmix32(fk ^ dv.hash_seed), dv.sets);
}
__device__ __forceinline__ int ways_in(const Dev& dv, uint32_t s) {
  const uint32_t lo = s * 32u;
  return dv.rows - lo >= 32u ? 32 : (int)(dv.rows - lo);
}
__device__ __forceinline__ uint32_t scr_hash(uint32_t fk) { return fmix32(fk * 0x9E3779B1u + 0x632BE5ABu); }
__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

__device__ __forceinline__ float4 ld_nc_v4(const float* p) {
  float4 v;
  asm volatile("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ uint32_t ld_nc_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint32_t ld_cg_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint4 ld_cg_v4u(const uint32_t* p) {
  uint4 v;
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_cg_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_v4(float* p, float4 v) {
  asm volatile("st.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w) : "memory");
}

// Copy the 32 rows named by the warp's lanes (src may be null = zero row; dst null =
// no store) for a compile-time row width D floats.  Loads for up to 8 float4 per
// lane are issued before any store.
template <int D>
__device__ __forceinline__ void gather_rows(const float* src, float* dst, int lane) {
  constexpr int VEC = D / 4;
  constexpr int LPR = VEC < 32 ? VEC : 32;  // lanes per row
  constexpr int RPP = 32 / LPR;             // rows per pass
  constexpr int VPL = VEC / LPR;            // float4 per lane per row
  constexpr int PASSES = 32 / RPP;
  constexpr int CH0 = (8 / VPL) > 0 ? (8 / VPL) : 1;
  constexpr int CH = CH0 < PASSES ? CH0 : PASSES;
  const int sub = lane % LPR, rs = lane / LPR;
#pragma unroll 1
  for (int p0 = 0; p0 < PASSES; p0 += CH) {
    float4 v[CH][VPL];
    float* o[CH];
#pragma unroll
    for (int q = 0; q < CH; ++q) {
      const int r = (p0 + q) * RPP + rs;
      const float* s = (const float*)__shfl_sync(kFull, (unsigned long long)src, r);
      o[q] = (float*)__shfl_sync(kFull, (unsigned long long)dst, r);
#pragma unroll
      for (int k = 0; k < VPL; ++k)
        v[q][k] = s ? ld_nc_v4(s + 4 * (sub + k * LPR)) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
#pragma unroll
    for (int q = 0; q < CH; ++q)
      if (o[q]) {
#pragma unroll
        for (int k = 0; k < VPL; ++k) st_v4(o[q] + 4 * (sub + k * LPR), v[q][k]);
      }
  }
}

// Fallback for warps whose lanes have different row widths or widths that are not a
// power of two: one row at a time, whole warp.
__device__ __forceinline__ void gather_rows_any(const float* src, float* dst, int d, int lane) {
#pragma unroll 1
  for (int r = 0; r < 32; ++r) {
    const float* s = (const float*)__shfl_sync(kFull, (unsigned long long)src, r);
    float* o = (float*)__shfl_sync(kFull, (unsigned long long)dst, r);
    const int dr = __shfl_sync(kFull, d, r);
    if (!o) continue;
    for (int c = lane; c < dr / 4; c += 32)
      st_v4(o + 4 * c, s ? ld_nc_v4(s + 4 * c) : make_float4(0.f, 0.f, 0.f, 0.f));
  }
}

// Rows of M misses held in registers across the warp (row r on lanes r*LPR..).
template <int D, int M>
struct RowBuf {
  static constexpr int VEC = D / 4;
  static constexpr int LPR = VEC < 32 ? VEC : 32;
  static constexpr int RPP = 32 / LPR;
  static constexpr int VPL = VEC / LPR;
  static constexpr int PASSES = (M + RPP - 1) / RPP;
  float4 v[PASSES][VPL];

  __device__ __forceinline__ void load(const float* src, int lane) {
    const int sub = lane % LPR, rs = lane / LPR;
#pragma unroll
    for (int p = 0; p < PASSES; ++p) {
      const int r = p * RPP + rs;
      const float* s = (const float*)__shfl_sync(kFull, (unsigned long long)src, r & 31);
#pragma unroll
      for (int k = 0; k < VPL; ++k)
        v[p][k] = (s && r < M) ? ld_nc_v4(s + 4 * (sub + k * LPR)) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
  }
  // store row r (for every r whose dst, held by lane r, is non-null)
  __device__ __forceinline__ void store(float* dst, int lane) const {
    const int sub = lane % LPR, rs = lane / LPR;
#pragma unroll
    for (int p = 0; p < PASSES; ++p) {
      const int r = p * RPP + rs;
      float* o = (float*)__shfl_sync(kFull, (unsigned long long)dst, r & 31);
      if (o && r < M) {
#pragma unroll
        for (int k = 0; k < VPL; ++k) st_v4(o + 4 * (sub + k * LPR), v[p][k]);
      }
    }
  }
};

template <int MAXT>
__global__ void __launch_bounds__(128) kq_kernel(const __grid_constant__ QArgs<MAXT> qa, const __grid_constant__ Dev dv) {
  __shared__ int64_t s_scan[MAXT + 1];
  __shared__ unsigned long long s_ctr[kNumCtr];
  for (int i = threadIdx.x; i <= qa.n; i += blockDim.x) s_scan[i] = qa.scan[i];
  if (threadIdx.x < kNumCtr) s_ctr[threadIdx.x] = 0;
  __syncthreads();

  const int lane = threadIdx.x & 31;
  const int64_t N = s_scan[qa.n];
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g - lane < N) {  // warp-uniform
    const uint32_t epoch = *(volatile uint32_t*)&dv.ctl->epoch;
    const bool active = g < N;

    // A1 self-identification: largest t with scan[t] <= g (reading R14)
    int t = 0;
    if (active) {
      int lo = 0, hi = qa.n;
      while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (s_scan[mid] <= g) lo = mid; else hi = mid;
      }
      t = lo;
    }
    const int64_t j = g - s_scan[t];
    const TableInfo* ti = dv.tables + t;
    const int64_t id = active ? qa.ids[t][j] : -1;
    const int64_t card = ti->card;
    const int d = ti->dim;

    // A2 re-encode to the flat key (size-aware code: fk = base_t + id)
    const bool valid = active && id >= 0 && id < card;
    const uint32_t fk = valid ? ti->base + (uint32_t)id : kEmpty;
    const uint32_t s = valid ? set_of(dv, fk) : 0u;

    // A3 probe: lane k holds way k of each of the warp's 32 sets (one 128 B line each)
    uint32_t kw[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      const uint32_t si = __shfl_sync(kFull, s, i);
      kw[i] = ld_nc_u32(dv.keys + (size_t)si * 32u + lane);
    }
    int way = -1;
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      const uint32_t fki = __shfl_sync(kFull, fk, i);
      const unsigned m = __ballot_sync(kFull, kw[i] == fki);
      if (lane == i && m) way = __ffs(m) - 1;
    }
    const bool hit = valid && way >= 0;
    const bool miss = valid && way < 0;
    const uint32_t slot = s * 32u + (uint32_t)way;
    const int64_t off = active ? qa.out_off[t] + j * (int64_t)d : 0;

    // A4 hit gather from the HBM slab (zero row for an invalid ID); misses are KM's
    const float* src = hit ? dv.slab + (size_t)slot * (size_t)d : nullptr;
    float* dst = (active && !miss) ? qa.out + off : nullptr;
    const int d0 = __shfl_sync(kFull, d, 0);
    const bool uni = __all_sync(kFull, !active || d == d0);
    if (uni && d0 == 32) gather_rows<32>(src, dst, lane);
    else if (uni && d0 == 64) gather_rows<64>(src, dst, lane);
    else if (uni && d0 == 128) gather_rows<128>(src, dst, lane);
    else if (uni && d0 == 16) gather_rows<16>(src, dst, lane);
    else if (uni && d0 == 8) gather_rows<8>(src, dst, lane);
    else if (uni && d0 == 256) gather_rows<256>(src, dst, lane);
    else gather_rows_any(src, dst, d, lane);

    // hit: refresh the way's timestamp once per batch (approximate LRU)
    bool uhit = false;
    if (hit) {
      const uint32_t old = ld_cg_u32(dv.ts + slot);
      if (old != epoch) uhit = atomicExch(dv.ts + slot, epoch) != epoch;
    }

    // A5 miss dedup: the lane whose CAS installs (epoch, fk) owns the miss
    int kind = 0;  // 1 = owner, 2 = duplicate
    uint32_t scr = 0;
    if (miss) {
      const unsigned long long tag = ((unsigned long long)epoch << 32) | fk;
      uint32_t h = scr_hash(fk) & dv.scr_mask;
      unsigned long long cur = ld_cg_u64(dv.scratch + h);
      while (true) {
        if (cur == tag) { kind = 2; break; }
        if ((uint32_t)(cur >> 32) != epoch) {
          const unsigned long long prev = atomicCAS(dv.scratch + h, cur, tag);
          if (prev == cur) { kind = 1; break; }
          cur = prev;
          continue;
        }
        h = (h + 1) & dv.scr_mask;
        cur = ld_cg_u64(dv.scratch + h);
      }
      scr = h;
    }

    const int par = epoch & 1u;
    const unsigned own_m = __ballot_sync(kFull, kind == 1);
    const unsigned dup_m = __ballot_sync(kFull, kind == 2);
    const unsigned lt = (1u << lane) - 1u;
    if (own_m) {
      uint32_t b = 0;
      if (lane == __ffs(own_m) - 1) b = atomicAdd(&dv.ctl->counts[par][0], (uint32_t)__popc(own_m));
      b = __shfl_sync(kFull, b, __ffs(own_m) - 1);
      if (kind == 1) {
        dv.miss[b + __popc(own_m & lt)] = MissRec{off, fk, scr, t, 0};
        // start the host-link transfer now: KM's loads of this row then hit L2
        if (dv.prefetch) {
          const float* hrow = ti->host + (size_t)id * (size_t)d;
          asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(hrow), "r"(4u * (unsigned)d) : "memory");
        }
      }
    }
    if (dup_m) {
      uint32_t b = 0;
      if (lane == __ffs(dup_m) - 1) b = atomicAdd(&dv.ctl->counts[par][1], (uint32_t)__popc(dup_m));
      b = __shfl_sync(kFull, b, __ffs(dup_m) - 1);
      if (kind == 2) {  // push onto the key's duplicate chain (epoch-tagged head)
        const uint32_t idx = b + __popc(dup_m & lt);
        unsigned long long old = ld_cg_u64(dv.dup_head + scr);
        while (true) {
          const uint32_t next = ((uint32_t)(old >> 32) == epoch) ? (uint32_t)old : 0u;
          dv.dup[idx] = DupRec{off, next, 0};
          const unsigned long long nw = ((unsigned long long)epoch << 32) | (idx + 1u);
          const unsigned long long prev = atomicCAS(dv.dup_head + scr, old, nw);
          if (prev == old) break;
          old = prev;
        }
      }
    }

    // A9 stats, warp-aggregated then block-aggregated
    const unsigned hm = __ballot_sync(kFull, hit), mm = __ballot_sync(kFull, miss);
    const unsigned im = __ballot_sync(kFull, active && !valid), um = __ballot_sync(kFull, uhit);
    if (lane == 0) {
      if (hm) atomicAdd(&s_ctr[C_HITS], (unsigned long long)__popc(hm));
      if (mm) atomicAdd(&s_ctr[C_MISSES], (unsigned long long)__popc(mm));
      if (im) {
        atomicAdd(&s_ctr[C_INVALID], (unsigned long long)__popc(im));
        dv.ctl->err_invalid = 1u;
      }
      if (um) atomicAdd(&s_ctr[C_UHITS], (unsigned long long)__popc(um));
      if (own_m) atomicAdd(&s_ctr[C_UMISS], (unsigned long long)__popc(own_m));
      if (dup_m) atomicAdd(&s_ctr[C_DUPS], (unsigned long long)__popc(dup_m));
    }
  }
  __syncthreads();
  if (threadIdx.x < kNumCtr && s_ctr[threadIdx.x])
    atomicAdd(dv.stats + (blockIdx.x % kStripes) * kNumCtr + threadIdx.x, s_ctr[threadIdx.x]);
}

// Victim way for flat key fk in its set: argmin (ts, key) over ways with ts < epoch,
// claimed by CAS(ts: old -> epoch).  Returns the slot, or -1 if every way of the set
// was read or written in this batch (epoch protection: bypass).  *old_key = the
// evicted key (kEmpty if the way was free).  One lane, 16 vector loads, no warp sync.
__device__ __forceinline__ int64_t claim_victim(const Dev& dv, uint32_t fk, uint32_t epoch, uint32_t* old_key) {
  const uint32_t s = set_of(dv, fk);
  const int nways = ways_in(dv, s);
  const uint32_t* kp = dv.keys + (size_t)s * 32u;
  uint32_t* tp = dv.ts + (size_t)s * 32u;
  while (true) {
    uint32_t kk[32], tt[32];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint4 a = ld_cg_v4u(kp + 4 * q), b = ld_cg_v4u(tp + 4 * q);
      kk[4 * q] = a.x; kk[4 * q + 1] = a.y; kk[4 * q + 2] = a.z; kk[4 * q + 3] = a.w;
      tt[4 * q] = b.x; tt[4 * q + 1] = b.y; tt[4 * q + 2] = b.z; tt[4 * q + 3] = b.w;
    }
    unsigned long long best = ~0ull;
    int bw = -1;
#pragma unroll
    for (int w = 0; w < 32; ++w) {
      const unsigned long long r = ((unsigned long long)tt[w] << 32) | kk[w];
      if (w < nways && tt[w] < epoch && r < best) { best = r; bw = w; }
    }
    if (bw < 0) return -1;
    if (atomicCAS(tp + bw, (uint32_t)(best >> 32), epoch) == (uint32_t)(best >> 32)) {
      *old_key = (uint32_t)best;
      return (int64_t)s * 32 + bw;
    }
  }
}

// KM for row width D: each warp iteration handles M unique misses.
template <int D, int M>
__device__ __forceinline__ void km_rows(const Dev& dv, float* __restrict__ out, uint32_t epoch, uint32_t nmiss,
                                        int lane, uint32_t gw, uint32_t nw, unsigned& ins, unsigned& ev,
                                        unsigned& byp, unsigned long long& hostb) {
  for (uint32_t base = gw * M; base < nmiss; base += nw * M) {
    const uint32_t k = base + lane;
    bool has = lane < M && k < nmiss;
    MissRec m{};
    const float* src = nullptr;
    if (has) {
      m = dv.miss[k];
      const TableInfo* ti = dv.tables + m.t;
      src = ti->host + (size_t)(m.fk - ti->base) * D;  // unified index: computed host address
    }
#ifdef FLECHE_EXPERIMENTS
    if (dv.exp_mode == 2) src = nullptr;  // timing experiment: no host loads
    if (dv.exp_mode == 1) has = false;    // timing experiment: loads only, no claim/store
#endif
    // A6: all of this warp's host-row loads go out now (zero-copy over the host link)
    RowBuf<D, M> rb;
    rb.load(src, lane);
    // A7 while they are in flight: admission + victim claim (L2 round trips only)
    float* slab_dst = nullptr;
    uint32_t fkey = kEmpty;
    if (has) {
      bool admit = true;
      if (!dv.admit_all)
        admit = splitmix64(dv.admit_seed ^ (uint64_t)m.fk ^ ((uint64_t)(epoch - 1u) << 32)) < dv.admit_thr;
      int64_t slot = -1;
      uint32_t old_key = kEmpty;
      if (admit) slot = claim_victim(dv, m.fk, epoch, &old_key);
      if (slot >= 0) {
        ++ins;
        if (old_key != kEmpty) ++ev;
        slab_dst = dv.slab + (size_t)slot * D;
        fkey = (uint32_t)slot;
      } else {
        ++byp;
      }
      hostb += 4ull * D;
    }
    // rows land: owner position, slab slot, then the key is published
    rb.store(has ? out + m.off : nullptr, lane);
    rb.store(slab_dst, lane);
    if (slab_dst) dv.keys[fkey] = m.fk;
    // A8 restore: walk each miss's duplicate chain
    uint32_t p = 0;
    if (has) {
      const unsigned long long h = ld_cg_u64(dv.dup_head + m.scr);
      p = ((uint32_t)(h >> 32) == epoch) ? (uint32_t)h : 0u;
    }
    while (__any_sync(kFull, p != 0)) {
      float* o = nullptr;
      if (p) {
        const DupRec r = dv.dup[p - 1];
        o = out + r.off;
        p = r.next;
      }
      rb.store(o, lane);
    }
  }
}

__global__ void __launch_bounds__(128) km_kernel(const __grid_constant__ Dev dv, float* __restrict__ out) {
  __shared__ unsigned long long s_ctr[kNumCtr];
  if (threadIdx.x < kNumCtr) s_ctr[threadIdx.x] = 0;
  __syncthreads();
  const uint32_t epoch = *(volatile uint32_t*)&dv.ctl->epoch;
  const int par = epoch & 1u;
  const uint32_t nmiss = *(volatile uint32_t*)&dv.ctl->counts[par][0];
  const int lane = threadIdx.x & 31;
  // block-interleaved warp numbering: consecutive miss chunks land on different SMs,
  // so the host-link loads of a batch are spread over the whole GPU
  const uint32_t gw = (threadIdx.x >> 5) * gridDim.x + blockIdx.x;
  const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
  unsigned ins = 0, ev = 0, byp = 0;
  unsigned long long hostb = 0;
#define FL_KM(D, M) km_rows<D, M>(dv, out, epoch, nmiss, lane, gw, nw, ins, ev, byp, hostb)
#define FL_KM_MS(D)                    \
  switch (dv.km_m) {                   \
    case 4: FL_KM(D, 4); break;        \
    case 16: FL_KM(D, 16); break;      \
    case 32: FL_KM(D, 32); break;      \
    default: FL_KM(D, 8); break;       \
  }
  switch (dv.dim) {  // fleche_create only admits these widths
    case 8: FL_KM_MS(8); break;
    case 16: FL_KM_MS(16); break;
    case 32: FL_KM_MS(32); break;
    case 64: FL_KM_MS(64); break;
    case 128: if (dv.km_m <= 4) FL_KM(128, 4); else FL_KM(128, 8); break;
    case 256: FL_KM(256, 4); break;
    default: break;
  }
#undef FL_KM_MS
#undef FL_KM
  ins = __reduce_add_sync(kFull, ins);
  ev = __reduce_add_sync(kFull, ev);
  byp = __reduce_add_sync(kFull, byp);
  for (int o = 16; o; o >>= 1) hostb += __shfl_xor_sync(kFull, hostb, o);
  if (lane == 0) {
    if (ins) atomicAdd(&s_ctr[C_INSERTED], (unsigned long long)ins);
    if (ev) atomicAdd(&s_ctr[C_EVICTED], (unsigned long long)ev);
    if (byp) atomicAdd(&s_ctr[C_BYPASSED], (unsigned long long)byp);
    if (hostb) atomicAdd(&s_ctr[C_HOSTBYTES], hostb);
  }
  __syncthreads();
  if (threadIdx.x < kNumCtr && s_ctr[threadIdx.x])
    atomicAdd(dv.stats + (blockIdx.x % kStripes) * kNumCtr + threadIdx.x, s_ctr[threadIdx.x]);
  if (threadIdx.x == 0) {
    const long long docc = (long long)s_ctr[C_INSERTED] - (long long)s_ctr[C_EVICTED];
    if (docc) atomicAdd((unsigned long long*)&dv.ctl->occ_rows, (unsigned long long)docc);
    __threadfence();
    const uint32_t prev = atomicAdd(&dv.ctl->done, 1u);
    if (prev == gridDim.x - 1) {  // last CTA: reset next batch's counters, advance the epoch
      dv.ctl->counts[par ^ 1][0] = 0;
      dv.ctl->counts[par ^ 1][1] = 0;
      dv.ctl->done = 0;
      __threadfence();
      *(volatile uint32_t*)&dv.ctl->epoch = epoch + 1u;
    }
  }
}

// Host-link probe: the miss-fetch access pattern (one row per lane, 16-byte vector
// loads, 32 rows per warp in flight) over seeded random rows of a mapped host buffer.
template <int D>
__global__ void __launch_bounds__(128) probe_host_kernel(const float* host, uint64_t span_rows, int64_t rows,
                                                         uint64_t seed, float* sink) {
  const int lane = threadIdx.x & 31;
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g - lane >= rows) return;
  const bool active = g < rows;
  const uint64_t r = splitmix64(seed + (uint64_t)g) % span_rows;
  const float* src = active ? host + r * (uint64_t)D : nullptr;
  float* dst = active ? sink + (size_t)(g & 4095) * D : nullptr;
  gather_rows<D>(src, dst, lane);
}

}  // namespace fl
