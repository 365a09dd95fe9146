// fleche.cu — host side of libfleche.so: the C ABI declared in include/fleche.h.
//
// Owns every device allocation (made once in fleche_create), the
// host-tier registration (pinned + mapped tables read by zero-copy loads,
// P:L855-860), per-call argument packing into kernel parameters (the Args Array and
// scan of P:L713-737 travel as __grid_constant__ parameters: no metadata copy on the
// query path), cross-stream ordering, and the stats read-back.
#include <cuda_runtime.h>

#include <immintrin.h>
#include <sys/prctl.h>
#include <time.h>

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <thread>
#include <vector>

#include "fleche.h"
#include "fns.h"

using namespace fl;

// Host-assisted miss fetch (FLECHE_FLAG_HOST_ASSIST; device side in kernels.cuh): the
// CPU-DRAM layer's threads gather the rows KQ requests into the pinned
// staging buffer.  Thread i owns every staging block k with k % nthreads == i, in every
// batch, so a block is only ever written by one thread, batch after batch in order: a
// thread that fell behind (its blocks timed out on the GPU, which fetched them itself)
// can never overwrite a newer batch's rows after their ready flag.
struct HostAssist {
  int nthreads = 0;
  std::vector<std::thread> th;
  std::atomic<bool> stop{false};
  // mapped pinned host memory (cudaHostAlloc): host pointers (the device sees the same
  // allocations through Dev::ha_*)
  void* mem = nullptr;
  HaReq* req = nullptr;                // [2][req_cap] (indexed like the miss list)
  HaDesc* desc = nullptr;              // [2]
  unsigned long long* bell = nullptr;  // doorbell (epoch): the descriptor of that batch is written
  unsigned long long* start = nullptr; // start word (epoch): KQ of that batch has begun
  uint32_t* ready = nullptr;           // [2][blk_cap] ready word of each staging block (= epoch once staged)
  uint32_t blk_cap = 0;
  uint32_t rbase[8] = {}, rcap[8] = {};  // staging rows of width class c: [rbase, rbase + rcap)
  float* stage = nullptr;              // [2][stage_floats]
  uint32_t req_cap = 0;
  bool nt_stores = true;  // FLECHE_HA_NT=0: plain memcpy into the staging buffer (A/B)
  bool stream = true;     // FLECHE_HA_STREAM=0: start on the doorbell, not on KQ's start word (A/B)
  uint64_t delay_ns = 0;  // FLECHE_HA_DELAY_US: fault injection (tests): each block is gathered this late
  uint64_t stage_floats = 0;
  // the tables as the host threads see them
  std::vector<const float*> host;
  std::vector<int64_t> card;
  std::vector<int32_t> dims;
#ifdef FLECHE_EXPERIMENTS
  uint64_t exp_t[64 * 2 * 64] = {};
  uint64_t* exp_pub = nullptr;  // CLOCK_REALTIME when each block's ready flag was published
  bool exp_nogather = getenv("FLECHE_HA_EXP_NOGATHER") != nullptr;
#endif
};

struct fleche_ctx {
  int device = 0;
  int n = 0;
  int max_dim = 0;
  int sm_count = 148;
  bool poisoned = false;
  int64_t max_lookups = 0;
  std::vector<int64_t> card;
  std::vector<int32_t> dims;
  std::vector<int32_t> cls;      // width class of each table
  std::vector<int32_t> cls_dim;  // row width of each class (ascending)
  std::vector<uint64_t> base;
  std::vector<int32_t> fbits;
  int key_bits = 0;
  bool lossy = false;            // short flat keys (R24): some tables hash their feature IDs
  std::vector<int32_t> hashed;   // per table
  uint64_t capacity_bytes = 0;
  uint64_t slab_floats = 0;
  std::vector<std::pair<void*, size_t>> registered;  // host ranges we registered
  Dev dv{};
  TableInfo* d_tables = nullptr;
  int km_blocks = 0;
  int km_bps = 4;  // KM CTAs per SM
  int kq_tma = 0;      // KQ's hit gather by bulk copies through shared memory (row width 32 or 64; 0 = registers)
  size_t kq_smem = 0;  // its dynamic shared memory (4 warps x 32 rows)
  int kf_ctas = 0;     // host-assisted early fetch: KQ CTAs that copy staged blocks into HBM (0 = off)
  int fwd_ctas = 0;    // host-assisted request forwarding: KQ CTAs that move requests to the host (0 = off)
  // ... from this many lookups per batch (FLECHE_HA_EARLY_MIN): a short KQ ends before the
  // host threads have staged much (cfg2, 213K lookups: 111 vs 106 us per batch without;
  // cfg5, 1.7M: 495 vs 570 us, profiles/)
  int64_t kf_min = 524288;
  bool per_table_launch = false;
  // decoupled hit copy (uniform layout): KG on a side stream, forked after KQ, joined after KM
  bool decoupled = false;
  cudaStream_t side = nullptr;
  cudaEvent_t fork_ev = nullptr, join_ev = nullptr;
  uint32_t* d_slots = nullptr;
  // lookups per batch from which the hit copy is decoupled (FLECHE_DECOUPLE_MIN): never by
  // default -- with the host-assisted miss fetch the fused copy measured faster at cfg2 (1780
  // vs 1728 Mkeys/s) and cfg5 (2604 vs 2551; profiles/bench_r02_decouple_*.json)
  int64_t decouple_min = INT64_MAX;
  size_t km_smem = 0;
  // host-side counters
  uint64_t batches = 0, lookups = 0, kernels = 0;
  // ordering across streams
  cudaStream_t last_stream = nullptr;
  bool have_last = false;
  cudaEvent_t chain_ev = nullptr;
  // fleche_query_host staging and pooled staging (lazy)
  int64_t* d_ids_stage = nullptr;
  float* d_out_stage = nullptr;
  float* d_out_stage2 = nullptr;   // fleche_query_host: second staging buffer (pipelined copies)
  cudaStream_t hq = nullptr, hd = nullptr;
  cudaEvent_t hq_ev[2] = {nullptr, nullptr}, hd_ev[2] = {nullptr, nullptr}, hc_ev[2] = {nullptr, nullptr};
  int hpar = 0;
  float* d_pool_stage = nullptr;
  uint64_t index_bytes = 0;
  // profiling (fleche_set_profiling)
  bool profiling = false;
  std::vector<cudaEvent_t> ev_pool;  // 3 or 4 per profiled query
  std::vector<int> ev_kinds;         // events recorded per profiled query (3 = one-hot, 4 = pooled)
  size_t ev_used = 0;
  // key-sharded mode (lazy): routing state and the last routed batch's geometry
  uint64_t* d_kdec = nullptr;
  RouteDev rd{};
  bool rd_ready = false;
  uint32_t repoch = 0;
  std::vector<int64_t> route_len;
  HostAssist* ha = nullptr;
  // watermark (full-scan) eviction (fleche_set_watermarks; reading R23)
  bool wm_on = false;
  long long wm_hi = 0, wm_lo = 0;
  unsigned long long* d_age_hist = nullptr;
  int ke_blocks = 0;
  PeerKeys route_peer{};         // fleche_route_p2p: owners' receive slots for this rank
  // fleche_prefill scratch output (lazy)
  float* d_prefill_out = nullptr;
  int64_t prefill_floats = 0;
};

namespace {

fleche_status poison(fleche_ctx* c, cudaError_t e, const char* what) {
  if (c) c->poisoned = true;
  fprintf(stderr, "[fleche] CUDA error in %s: %s\n", what, cudaGetErrorString(e));
  return FLECHE_ECUDA;
}

#define FL_CUDA(ctx, call)                                   \
  do {                                                       \
    cudaError_t e_ = (call);                                 \
    if (e_ != cudaSuccess) return poison((ctx), e_, #call);  \
  } while (0)

int ceil_log2_u64(int64_t c) {
  int f = 0;
  while (f < 63 && (int64_t(1) << f) < c) ++f;
  return f;
}

// Size-aware coding (R3): larger tables get shorter table IDs.
// feature bits f_t = max(1, ceil(log2 c_t)); table IDs assigned as a canonical prefix
// code in order of increasing length; fk = base_t + id.  Returns B_min or -1 if the
// code plus the reserved all-ones key does not fit in 32 bits.
int size_aware_code(const std::vector<int64_t>& card, std::vector<uint64_t>& base, std::vector<int32_t>& fb) {
  const int n = (int)card.size();
  fb.resize(n);
  base.resize(n);
  unsigned __int128 span = 1;  // the EMPTY key
  for (int t = 0; t < n; ++t) {
    fb[t] = std::max(1, ceil_log2_u64(card[t]));
    span += (unsigned __int128)1 << fb[t];
  }
  int bmin = 0;
  while (((unsigned __int128)1 << bmin) < span) ++bmin;
  if (bmin > 32) return -1;
  std::vector<int> idx(n);
  for (int t = 0; t < n; ++t) idx[t] = t;
  std::sort(idx.begin(), idx.end(), [&](int a, int b) { return fb[a] != fb[b] ? fb[a] > fb[b] : a < b; });
  uint64_t at = 0;
  for (int t : idx) {
    base[t] = at;
    at += uint64_t(1) << fb[t];
  }
  return bmin;
}

// Short flat keys (key_bits < B_min, reading R24): tables in
// ascending size keep their exact 2^f_t codes while every remaining table can still get
// one code; the space left is shared by the remaining tables in proportion to their
// sizes (power-of-two blocks, 2^g * C <= R * c_t, g < f_t), their feature IDs hashed
// into g bits; if the one-code floor overflows the space, the largest block is halved
// (ties: the later table in ascending order) until it fits.  Canonical layout as in
// size_aware_code.  Returns the number of hashed tables, -1 if impossible.
int short_code(const std::vector<int64_t>& card, int B, std::vector<uint64_t>& base, std::vector<int32_t>& bits,
               std::vector<int32_t>& hashed) {
  const int n = (int)card.size();
  using u128 = unsigned __int128;
  const u128 space = ((u128)1 << B) - 1;  // the all-ones key stays EMPTY
  std::vector<int> f(n), up(n);
  for (int t = 0; t < n; ++t) f[t] = std::max(1, ceil_log2_u64(card[t]));
  for (int t = 0; t < n; ++t) up[t] = t;
  std::stable_sort(up.begin(), up.end(), [&](int a, int b) { return card[a] < card[b]; });
  int keep = 0;
  u128 acc = 0;
  for (int i = 0; i <= n; ++i) {
    if (acc + (u128)(n - i) <= space) keep = i;
    if (i < n) acc += (u128)1 << f[up[i]];
  }
  u128 left = space, rest = 0;
  for (int i = 0; i < keep; ++i) left -= (u128)1 << f[up[i]];
  for (int i = keep; i < n; ++i) rest += (u128)card[up[i]];
  bits.assign(n, 0);
  hashed.assign(n, 0);
  for (int i = 0; i < n; ++i) {
    const int t = up[i];
    if (i < keep) {
      bits[t] = f[t];
      continue;
    }
    hashed[t] = 1;
    int g = 0;
    while (g + 1 < f[t] && ((u128)1 << (g + 1)) * rest <= left * (u128)card[t]) ++g;
    bits[t] = g;
  }
  for (;;) {
    u128 tot = 0;
    int big = -1;
    for (int i = keep; i < n; ++i) {
      tot += (u128)1 << bits[up[i]];
      if (bits[up[i]] > 0 && (big < 0 || bits[up[i]] >= bits[up[big]])) big = i;
    }
    if (tot <= left) break;
    if (big < 0) return -1;
    bits[up[big]]--;
  }
  std::vector<int> ord(n);
  for (int t = 0; t < n; ++t) ord[t] = t;
  std::stable_sort(ord.begin(), ord.end(), [&](int a, int b) { return bits[a] > bits[b]; });
  base.assign(n, 0);
  uint64_t at = 0;
  for (int t : ord) {
    base[t] = at;
    at += uint64_t(1) << bits[t];
  }
  return n - keep;
}

uint32_t next_pow2(uint64_t x) {
  uint64_t p = 1;
  while (p < x) p <<= 1;
  return (uint32_t)p;
}

bool valid_dim(int d) { return d == 8 || d == 16 || d == 32 || d == 64 || d == 128 || d == 256; }

// Page-lock and map the caller's tables.  Ranges that touch a common page are
// registered together (tables usually share one allocation; a page can be
// registered only once).
fleche_status register_host(fleche_ctx* c, const float* const* host, std::vector<const float*>& dev_ptrs) {
  const uintptr_t pg = 4096;
  std::vector<std::pair<uintptr_t, uintptr_t>> r;
  for (int t = 0; t < c->n; ++t) {
    uintptr_t a = (uintptr_t)host[t], b = a + (size_t)c->card[t] * (size_t)c->dims[t] * 4u;
    r.push_back({a, b});
  }
  std::sort(r.begin(), r.end());
  std::vector<std::pair<uintptr_t, uintptr_t>> m;
  for (auto& x : r) {
    if (!m.empty() && (x.first & ~(pg - 1)) <= ((m.back().second - 1) & ~(pg - 1)))
      m.back().second = std::max(m.back().second, x.second);
    else
      m.push_back(x);
  }
  for (auto& x : m) {
    void* p = (void*)x.first;
    cudaPointerAttributes at{};
    if (cudaPointerGetAttributes(&at, p) == cudaSuccess && at.type == cudaMemoryTypeHost) continue;  // pinned already
    cudaGetLastError();
    cudaError_t e = cudaHostRegister(p, x.second - x.first, cudaHostRegisterMapped | cudaHostRegisterPortable);
    if (e == cudaErrorHostMemoryAlreadyRegistered) {
      cudaGetLastError();
      continue;
    }
    if (e != cudaSuccess) return poison(c, e, "cudaHostRegister");
    c->registered.push_back({p, x.second - x.first});
  }
  dev_ptrs.resize(c->n);
  for (int t = 0; t < c->n; ++t) {
    void* dp = nullptr;
    FL_CUDA(c, cudaHostGetDevicePointer(&dp, (void*)host[t], 0));
    dev_ptrs[t] = (const float*)dp;
  }
  return FLECHE_OK;
}

// Row copy into the staging buffer with non-temporal stores: the rows go to DRAM, not
// into this core's cache, so the GPU's link reads of them are not stalled snooping
// modified lines out of the writer's cache (dst 32 B aligned, bytes a multiple of 32).
__attribute__((target("avx2"))) void stage_row(float* dst, const float* src, size_t bytes) {
  for (size_t b = 0; b < bytes; b += 32)
    _mm256_stream_si256((__m256i*)((char*)dst + b), _mm256_loadu_si256((const __m256i*)((const char*)src + b)));
}

// One host-assist thread: the CPU-DRAM layer queried while the batch is still being
// indexed (Fig 8b).  KQ's first CTA writes the batch's epoch to the start word
// when it begins; from then on the thread streams its staging blocks (block k = staging
// rows [64k, 64k + 64), k % nthreads == me, increasing k within each width class): KQ
// hands out a class's staging rows in the order it discovers the misses, so block k's
// requests arrive while later misses are still being found.  Each row is gathered as soon
// as its request carries this batch's tags, with non-temporal stores, and a block's ready
// word (= epoch) is published once its rows are in place -- a full block at once, the
// class's last partial block once the doorbell descriptor (written by KQ's last CTA) gives
// the class's count.  Blocks past the descriptor's host share (hcut) are not started; a
// block gathered before the descriptor arrived and then left to KM's zero-copy share is
// simply not read.  Spins while batches keep coming; after ~20 ms without progress it
// polls every 20 us (an idle ctx burns no core).  No `pause` in the spin: on a KVM guest
// it can trigger pause-loop exits that deschedule the vCPU.
void ha_worker(HostAssist* h, int me) {
  prctl(PR_SET_TIMERSLACK, 1000UL, 0, 0, 0);  // idle polls wake within ~20 us, not the default 50 us slack
  auto now_ns = []() {
    struct timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (uint64_t)ts.tv_sec * 1000000000ull + (uint64_t)ts.tv_nsec;
  };
  auto idle = [&](uint64_t since) {  // back off after 20 ms without anything to do
    if (now_ns() - since > 20000000ull) {
      struct timespec ts = {0, 20000};
      nanosleep(&ts, nullptr);
    }
  };
  const int nt = (int)h->host.size();
  const uint64_t T = (uint64_t)h->nthreads;
  uint32_t last = 0;
  uint64_t t_last = now_ns();
  uint64_t spins = 0;
  // FLECHE_HA_STREAM=0: wait for the doorbell (every request written) instead of the start word
  const unsigned long long* wake = h->stream ? h->start : h->bell;
  while (!h->stop.load(std::memory_order_relaxed)) {
    const uint32_t e = (uint32_t)__atomic_load_n(wake, __ATOMIC_ACQUIRE);
    if (e == last) {
      if ((++spins & 1023) == 0) idle(t_last);
      continue;
    }
    last = e;
    t_last = now_ns();
#ifdef FLECHE_EXPERIMENTS
    auto rt = []() {
      struct timespec ts;
      clock_gettime(CLOCK_REALTIME, &ts);
      return (uint64_t)ts.tv_sec * 1000000000ull + (uint64_t)ts.tv_nsec;
    };
    if (me < 64) h->exp_t[(e % 64) * 128 + me] = rt();
#endif
    const int par = e & 1u;
    uint32_t* ready = h->ready + (size_t)par * h->blk_cap;
    const volatile HaReq* rq = h->req + (size_t)par * h->req_cap;
    float* st = h->stage + (size_t)par * h->stage_floats;
    // the doorbell descriptor of this batch (written without a system fence: accepted once
    // both epoch fields carry this batch and a second read agrees)
    HaDesc d;
    bool have_d = false;
    uint64_t t_d = 0;
    auto poll_desc = [&]() {
      if (have_d) return;
      HaDesc a, b2;
      memcpy(&a, (const void*)(h->desc + par), sizeof a);
      __atomic_thread_fence(__ATOMIC_ACQUIRE);
      memcpy(&b2, (const void*)(h->desc + par), sizeof b2);
      if (a.epoch == e && a.epoch2 == e && !memcmp(&a, &b2, sizeof a)) {
        d = a;
        have_d = true;
        t_d = now_ns();
      }
    };
    // request i of this batch, if it has arrived (KQ wrote it without a system fence: each
    // 8-byte half is written and read whole, and both carry this batch's tags, so a request
    // still in flight -- or a read that caught only one half -- is never taken)
    auto fetch = [&](uint64_t i, HaReq* out) -> bool {
      HaReq a{rq[i].tid, rq[i].stage};
      if (!ha_req_current(a, e)) return false;
      *out = a;
      return true;
    };
    auto src_of = [&](const HaReq& r, int32_t* dim, uint64_t* so) -> const float* {
      const int t = (int)(r.tid >> 55);
      const int64_t id = (int64_t)(r.tid & kReqLow40);
      *so = r.stage & kReqLow40;
      if (*so == kReqLow40 || t >= nt || id >= h->card[t]) return nullptr;  // no room / defensive
      *dim = h->dims[t];
      if (*so + (uint64_t)*dim > h->stage_floats) return nullptr;
      return h->host[t] + (size_t)id * (size_t)*dim;
    };
    // static ownership (staging block b belongs to thread b % nthreads in every batch, taken
    // in increasing b): a thread that stalls past the GPU's give-up can only ever overwrite
    // its own blocks, which it republishes only after rewriting them
    struct Cursor {
      uint64_t kb = 0, i = 0;  // current block, next row
      bool done = true;
    } cur[8];
    for (int c = 0; c < 8; ++c) {
      if (!h->rcap[c]) continue;
      const uint64_t kb0 = h->rbase[c] / kHaBlock;
      cur[c].kb = kb0 + (T - kb0 % T + (uint64_t)me) % T;
      cur[c].i = cur[c].kb * kHaBlock;
      cur[c].done = cur[c].i >= (uint64_t)h->rbase[c] + h->rcap[c];
    }
    uint64_t t_prog = now_ns();
    bool delayed = false;  // fault injection: once per block
    while (true) {
      poll_desc();
      bool all_done = true, progressed = false;
      for (int c = 0; c < 8; ++c) {
        Cursor& q = cur[c];
        if (q.done) continue;
        const uint64_t rb = h->rbase[c], lo = q.kb * kHaBlock;
        uint64_t hi = std::min<uint64_t>(lo + kHaBlock, rb + h->rcap[c]);
        if (have_d) {  // the batch's count and the host share are known
          const uint64_t nrow = std::min<uint64_t>(d.cnt[c], h->rcap[c]);
          if (q.kb - rb / kHaBlock >= d.hcut[c] || lo >= rb + nrow) {
            q.done = true;
            continue;
          }
          hi = std::min<uint64_t>(hi, rb + nrow);
        }
        all_done = false;
        if (h->delay_ns && !delayed) {  // a stalled host thread (tests): its blocks time out on the GPU
          struct timespec ts = {(time_t)(h->delay_ns / 1000000000ull), (long)(h->delay_ns % 1000000000ull)};
          nanosleep(&ts, nullptr);
          delayed = true;
        }
        constexpr uint64_t PF = 12;  // rows prefetched ahead (~4 lines each: keeps the line fill buffers busy)
        for (; q.i < hi; ++q.i) {
          HaReq r;
          if (!fetch(q.i, &r)) break;  // not arrived yet
          if (q.i + PF < hi) {
            HaReq r2;
            int32_t d2 = 0;
            uint64_t so2 = 0;
            const float* p2 = fetch(q.i + PF, &r2) ? src_of(r2, &d2, &so2) : nullptr;
            if (p2)
              for (int b = 0; b < d2 * 4; b += 64) __builtin_prefetch((const char*)p2 + b, 0, 0);
          }
          int32_t dd = 0;
          uint64_t so = 0;
          if (const float* p = src_of(r, &dd, &so)) {
#ifdef FLECHE_EXPERIMENTS
            if (!h->exp_nogather)  // timing experiment: publish without gathering (wrong rows)
#endif
            {
              if (h->nt_stores) stage_row(st + so, p, (size_t)dd * 4u);
              else memcpy(st + so, p, (size_t)dd * 4u);
            }
          }
          progressed = true;
        }
        if (q.i == hi && (hi == lo + kHaBlock || have_d)) {  // the block is complete
          if (h->nt_stores) _mm_sfence();  // streaming stores are weakly ordered: drain them before the ready word
          __atomic_store_n(ready + q.kb, e, __ATOMIC_RELEASE);
#ifdef FLECHE_EXPERIMENTS
          if (h->exp_pub) {
            struct timespec ts;
            clock_gettime(CLOCK_REALTIME, &ts);
            h->exp_pub[q.kb] = (uint64_t)ts.tv_sec * 1000000000ull + (uint64_t)ts.tv_nsec;
          }
#endif
          q.kb += T;
          q.i = q.kb * kHaBlock;
          q.done = q.i >= rb + h->rcap[c];
          delayed = false;
          progressed = true;
        }
      }
      if (all_done || h->stop.load(std::memory_order_relaxed)) break;
      const uint64_t now = now_ns();
      if (progressed) {
        t_prog = now;
        continue;
      }
      // waiting for requests: give up on this batch when a newer one has started, or when a
      // request never arrived ~1 ms after the descriptor (KM's poller times out and reads
      // those blocks zero-copy)
      if ((uint32_t)__atomic_load_n(wake, __ATOMIC_ACQUIRE) != e) break;
      if (have_d && now - std::max(t_d, t_prog) > 1000000ull) break;
      if ((++spins & 1023) == 0) idle(t_prog);
    }
    t_last = now_ns();
#ifdef FLECHE_EXPERIMENTS
    if (me < 64) h->exp_t[(e % 64) * 128 + 64 + me] = rt();
#endif
  }
}

void ha_stop(HostAssist* h) {
  if (!h) return;
  h->stop.store(true);
  for (auto& t : h->th)
    if (t.joinable()) t.join();
  h->th.clear();
  if (h->mem) cudaFreeHost(h->mem);
  h->mem = nullptr;
}

void free_all(fleche_ctx* c) {
  void* ptrs[] = {c->dv.keys, c->dv.ts, c->dv.loc, c->dv.lock, c->dv.slab, c->dv.scratch, c->dv.owner_off,
                  c->dv.firstpos, c->dv.ipos,
                  c->dv.miss, c->dv.dup, c->dv.ctl, c->dv.stats, c->d_tables, c->d_ids_stage, c->d_out_stage,
                  c->d_pool_stage, c->d_kdec, c->rd.scratch, c->rd.slotval, c->rd.inv, c->rd.region, c->rd.cnt,
                  c->rd.prefix, c->rd.done, c->rd.stats, c->d_slots, c->d_age_hist, c->d_prefill_out,
                  c->d_out_stage2, c->dv.ha_seen, c->dv.ha_hstage, c->dv.ha_hseen, c->dv.ha_reqd};
  for (void* p : ptrs)
    if (p) cudaFree(p);
  for (auto& r : c->registered) cudaHostUnregister(r.first);
  c->registered.clear();
  if (c->chain_ev) cudaEventDestroy(c->chain_ev);
  if (c->fork_ev) cudaEventDestroy(c->fork_ev);
  if (c->join_ev) cudaEventDestroy(c->join_ev);
  for (int i = 0; i < 2; ++i) {
    if (c->hq_ev[i]) cudaEventDestroy(c->hq_ev[i]);
    if (c->hd_ev[i]) cudaEventDestroy(c->hd_ev[i]);
    if (c->hc_ev[i]) cudaEventDestroy(c->hc_ev[i]);
  }
  if (c->hq) cudaStreamDestroy(c->hq);
  if (c->hd) cudaStreamDestroy(c->hd);
  if (c->side) cudaStreamDestroy(c->side);
  for (cudaEvent_t e : c->ev_pool) cudaEventDestroy(e);
  c->ev_pool.clear();
  if (c->ha) {
    ha_stop(c->ha);
    delete c->ha;
    c->ha = nullptr;
  }
}

fleche_status ensure_device(fleche_ctx* c) {
  int cur = -1;
  if (cudaGetDevice(&cur) != cudaSuccess || cur != c->device) FL_CUDA(c, cudaSetDevice(c->device));
  return FLECHE_OK;
}

// Calls on one ctx run in call order even across streams.
fleche_status order_on(fleche_ctx* c, cudaStream_t s) {
  if (c->have_last && s != c->last_stream) {
    FL_CUDA(c, cudaEventRecord(c->chain_ev, c->last_stream));
    FL_CUDA(c, cudaStreamWaitEvent(s, c->chain_ev, 0));
  }
  c->last_stream = s;
  c->have_last = true;
  return FLECHE_OK;
}

fleche_status prof_event(fleche_ctx* c, cudaStream_t s, bool first, int kinds) {
  if (!c->profiling) return FLECHE_OK;
  if (c->ev_pool.size() <= c->ev_used) {
    cudaEvent_t e;
    FL_CUDA(c, cudaEventCreate(&e));
    c->ev_pool.push_back(e);
  }
  if (first) c->ev_kinds.push_back(kinds);
  FL_CUDA(c, cudaEventRecord(c->ev_pool[c->ev_used++], s));
  return FLECHE_OK;
}

// Launch with programmatic stream serialization (PDL): the kernel's launch and prologue
// overlap its predecessor's tail; the kernel's pdl_wait() orders its dependent work.
// Per-kernel PDL mask (bit 0 KQ, 2 the watermark scan, 3 KP).  KM is a cooperative launch
// (never PDL): its grid barrier needs every CTA resident, and its early placement during
// KQ's tail measured slower for the address-ordered miss fetch anyway (profiles/README.md).
enum { kPdlKQ = 0, kPdlKM = 1, kPdlKD = 2, kPdlKP = 3, kPdlNone = 30, kPdlCoop = 31 };
int pdl_mask() {
  static const int m = getenv("FLECHE_NO_PDL") ? 0 : (getenv("FLECHE_PDL_MASK") ? atoi(getenv("FLECHE_PDL_MASK")) : 0xD);
  return m;
}
template <typename... KArgs, typename... Args>
cudaError_t launch_k(int which, void (*kern)(KArgs...), unsigned grid, unsigned block, size_t smem, cudaStream_t s,
                     Args&&... args) {
  const bool g_pdl = which != kPdlCoop && ((pdl_mask() >> which) & 1);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  if (which == kPdlCoop) {  // every CTA resident at once (KM2's grid barrier)
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
  } else {
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
  }
  cfg.attrs = attr;
  cfg.numAttrs = (g_pdl || which == kPdlCoop) ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// The miss side of one batch: KM (fetch + insert + restore), a cooperative launch (its grid
// barrier before the restore needs every CTA resident; km_blocks never exceeds that).
void launch_miss(fleche_ctx* c, cudaStream_t s, const KMArgs& ka) {
  static const bool coop = !(getenv("FLECHE_KM_COOP") && !atoi(getenv("FLECHE_KM_COOP")));  // A/B of the launch cost only
  launch_k(coop ? kPdlCoop : kPdlKM, km_fn(c->dv.bytes != 0, c->cls_dim.size() == 1 ? c->max_dim : 0), c->km_blocks, 128, c->km_smem, s,
           c->dv, ka);
  c->kernels += 1;
}

// Watermark scan after a batch's KM (fleche_set_watermarks): KE1 + KE2, both exit at
// once when the cached bytes are <= hi.
void launch_scan(fleche_ctx* c, cudaStream_t s) {
  if (!c->wm_on) return;
  KEArgs ea{c->d_age_hist, c->wm_hi, c->wm_lo};
  launch_k(kPdlKD, ke_hist_fn(), c->ke_blocks, 256, 0, s, c->dv, ea);
  launch_k(kPdlKD, ke_evict_fn(), c->ke_blocks, 256, 0, s, c->dv, ea);
  c->kernels += 2;
}

// KQ + KM for one batch of one-hot lookups into `out` (table-major rows).
template <int MAXT>
fleche_status launch_query(fleche_ctx* c, const int64_t* const* ids, const int64_t* lengths, float* out,
                           cudaStream_t s, int64_t total, int nev) {
  QArgs<MAXT> qa;
  memset(&qa, 0, sizeof(qa));
  qa.n = c->n;
  qa.out = out;
  KMArgs ka;
  memset(&ka, 0, sizeof(ka));
  ka.out = out;
  ka.ncls = (int)c->cls_dim.size();
  int64_t cls_len[8] = {0};
  int64_t acc = 0, oacc = 0;
  for (int t = 0; t < c->n; ++t) {
    qa.ids[t] = ids[t];
    qa.scan[t] = acc;
    qa.out_off[t] = oacc;
    acc += lengths[t];
    oacc += lengths[t] * (int64_t)c->dims[t];
    cls_len[c->cls[t]] += lengths[t];
  }
  qa.scan[c->n] = acc;
  int64_t coff = 0;  // each width's region of the miss list: at most its lookups
  for (int k = 0; k < ka.ncls; ++k) {
    qa.cls_off[k] = ka.cls_off[k] = coff;
    ka.cls_dim[k] = c->cls_dim[k];
    coff += cls_len[k];
  }
  fleche_status st = prof_event(c, s, true, nev);
  if (st != FLECHE_OK) return st;
  // small batches: the fork/join costs more than the overlap saves (cfg1 measured +5 %)
  const bool decouple = c->decoupled && total >= c->decouple_min && !c->per_table_launch;
  if (decouple) qa.slots = c->d_slots;
  // host-assisted: KQ's last CTA rings the host threads' doorbell (FLECHE_HA_BELL=km: KM does)
  static const bool bell_km = getenv("FLECHE_HA_BELL") && !strcmp(getenv("FLECHE_HA_BELL"), "km");
  qa.ha_bell = c->dv.ha && !bell_km;
  ka.bell = c->dv.ha && bell_km;
  qa.ncls = ka.ncls;
  for (int k = 0; k < ka.ncls; ++k) qa.cls_dim[k] = c->cls_dim[k];
  if (total > 0 && !c->per_table_launch) {
    qa.nfetch = (qa.ha_bell && !decouple && total >= c->kf_min) ? c->kf_ctas : 0;
    qa.nfwd = (qa.ha_bell && c->dv.ha_reqd) ? c->fwd_ctas : 0;
    const int64_t blocks = (total + FL_KQ_THREADS - 1) / FL_KQ_THREADS + qa.nfetch + qa.nfwd;
    launch_k(kPdlKQ, kq_fn<MAXT>(c->kq_tma), (unsigned)blocks, FL_KQ_THREADS, c->kq_smem, s, qa, c->dv);
    c->kernels++;
    if (decouple) {  // fork: the hit copy runs on the side stream, concurrently with KM
      FL_CUDA(c, cudaEventRecord(c->fork_ev, s));
      FL_CUDA(c, cudaStreamWaitEvent(c->side, c->fork_ev, 0));
      launch_k(kPdlNone, kg_fn<MAXT>(), (unsigned)blocks, 128, 0, c->side, qa, c->dv);
      c->kernels++;
      FL_CUDA(c, cudaEventRecord(c->join_ev, c->side));
    }
  } else if (total > 0) {  // ablation: one query launch per table (n launches)
    QArgs<32> q1;
    memset(&q1, 0, sizeof(q1));
    q1.n = 1;
    q1.out = out;
    for (int k = 0; k < 8; ++k) q1.cls_off[k] = qa.cls_off[k];
    for (int t = 0; t < c->n; ++t) {
      if (lengths[t] == 0) continue;
      q1.t0 = t;
      q1.g0 = qa.scan[t];
      q1.ids[0] = ids[t];
      q1.scan[0] = 0;
      q1.scan[1] = lengths[t];
      q1.out_off[0] = qa.out_off[t];
      launch_k(kPdlKQ, kq_fn<32>(c->kq_tma), (unsigned)((lengths[t] + FL_KQ_THREADS - 1) / FL_KQ_THREADS), FL_KQ_THREADS,
               c->kq_smem, s, q1, c->dv);
      c->kernels++;
    }
  }
  if ((st = prof_event(c, s, false, 0)) != FLECHE_OK) return st;
  launch_miss(c, s, ka);
  if ((st = prof_event(c, s, false, 0)) != FLECHE_OK) return st;  // (the former KD's slot: empty)
  if (decouple) FL_CUDA(c, cudaStreamWaitEvent(s, c->join_ev, 0));  // join: out complete on s
  launch_scan(c, s);
  if ((st = prof_event(c, s, false, 0)) != FLECHE_OK) return st;
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return poison(c, e, "kernel launch");
  return FLECHE_OK;
}

fleche_status query_impl(fleche_ctx* c, const int64_t* const* ids, const int64_t* lengths, float* out,
                         cudaStream_t s, int nev = 4) {
  int64_t total = 0;
  for (int t = 0; t < c->n; ++t) {
    if (lengths[t] < 0) return FLECHE_EINVAL;
    if (lengths[t] > 0 && !ids[t]) return FLECHE_EINVAL;
    total += lengths[t];
  }
  if (total > c->max_lookups) return FLECHE_EINVAL;
  if (total > 0 && (!out || ((uintptr_t)out & 15u))) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  st = order_on(c, s);
  if (st != FLECHE_OK) return st;
  if (c->n <= 32) st = launch_query<32>(c, ids, lengths, out, s, total, nev);
  else if (c->n <= 128) st = launch_query<128>(c, ids, lengths, out, s, total, nev);
  else st = launch_query<FLECHE_MAX_TABLES>(c, ids, lengths, out, s, total, nev);
  if (st == FLECHE_OK) {
    c->batches++;
    c->lookups += (uint64_t)total;
  }
  return st;
}

template <int MAXT>
fleche_status launch_pool(fleche_ctx* c, const int64_t* const* offsets, const int64_t* bags, const int64_t* nnz,
                          float* out, cudaStream_t s) {
  PArgs<MAXT> pa;
  memset(&pa, 0, sizeof(pa));
  pa.n = c->n;
  pa.stage = c->d_pool_stage;
  pa.out = out;
  int64_t cs = 0, so = 0, oo = 0;
  for (int t = 0; t < c->n; ++t) {
    pa.offs[t] = offsets[t];
    pa.cscan[t] = cs;
    pa.stage_off[t] = so;
    pa.out_off[t] = oo;
    cs += bags[t] * (int64_t)(c->dims[t] / 4);
    so += nnz[t] * (int64_t)c->dims[t];
    oo += bags[t] * (int64_t)c->dims[t];
  }
  pa.cscan[c->n] = cs;
  if (cs > 0) {
    launch_k(kPdlKP, kp_fn<MAXT>(), (unsigned)((cs + 255) / 256), 256, 0, s, pa, (const TableInfo*)c->d_tables);
    c->kernels++;
  }
  fleche_status st = prof_event(c, s, false, 0);
  if (st != FLECHE_OK) return st;
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return poison(c, e, "kernel launch");
  return FLECHE_OK;
}

}  // namespace

extern "C" {

const char* fleche_strerror(fleche_status s) {
  switch (s) {
    case FLECHE_OK: return "ok";
    case FLECHE_EINVAL: return "invalid argument";
    case FLECHE_ENOMEM: return "out of memory";
    case FLECHE_ECUDA: return "CUDA error";
    case FLECHE_ENCCL: return "NCCL error";
    case FLECHE_ERANGE: return "an ID outside [0, c_t) was looked up";
    case FLECHE_ESTATE: return "context poisoned by an earlier CUDA error";
  }
  return "unknown status";
}

fleche_status fleche_create(const fleche_config* cfg, fleche_ctx** out) {
  if (!cfg || !out) return FLECHE_EINVAL;
  *out = nullptr;
  const int n = cfg->num_tables;
  if (n < 1 || n > FLECHE_MAX_TABLES || !cfg->cardinalities || !cfg->dims || !cfg->host_tables) return FLECHE_EINVAL;
  const uint32_t known = FLECHE_FLAG_STATIC_PER_TABLE | FLECHE_FLAG_PER_TABLE_LAUNCH |
                         FLECHE_FLAG_HOST_ASSIST | FLECHE_FLAG_FUSED_HIT_COPY | FLECHE_FLAG_NO_HOST_ASSIST;
  if (cfg->max_lookups < 1 || cfg->max_lookups > (int64_t(1) << 31) || (cfg->flags & ~known) || cfg->reserved)
    return FLECHE_EINVAL;
  if ((cfg->flags & FLECHE_FLAG_HOST_ASSIST) &&
      (cfg->flags & (FLECHE_FLAG_PER_TABLE_LAUNCH | FLECHE_FLAG_NO_HOST_ASSIST)))
    return FLECHE_EINVAL;
  for (int t = 0; t < n; ++t) {
    if (cfg->cardinalities[t] < 1 || !valid_dim(cfg->dims[t])) return FLECHE_EINVAL;
    if (!cfg->host_tables[t] || ((uintptr_t)cfg->host_tables[t] & 15u)) return FLECHE_EINVAL;
  }
  fleche_ctx* c = new (std::nothrow) fleche_ctx();
  if (!c) return FLECHE_ENOMEM;
  c->device = cfg->device;
  c->n = n;
  c->max_lookups = cfg->max_lookups;
  c->card.assign(cfg->cardinalities, cfg->cardinalities + n);
  c->dims.assign(cfg->dims, cfg->dims + n);
  c->key_bits = size_aware_code(c->card, c->base, c->fbits);
  c->hashed.assign(n, 0);
  if (cfg->key_bits < 0 || cfg->key_bits > 32) {
    delete c;
    return FLECHE_EINVAL;
  }
  if (cfg->key_bits > 0 && (c->key_bits < 0 || cfg->key_bits < c->key_bits)) {  // short flat keys (R24)
    if (short_code(c->card, cfg->key_bits, c->base, c->fbits, c->hashed) < 0) {
      delete c;
      return FLECHE_EINVAL;
    }
    c->key_bits = cfg->key_bits;
    c->lossy = true;
  }
  for (int t = 0; t < n; ++t)
    if (std::find(c->cls_dim.begin(), c->cls_dim.end(), c->dims[t]) == c->cls_dim.end()) c->cls_dim.push_back(c->dims[t]);
  std::sort(c->cls_dim.begin(), c->cls_dim.end());
  c->cls.resize(n);
  for (int t = 0; t < n; ++t)
    c->cls[t] = (int)(std::find(c->cls_dim.begin(), c->cls_dim.end(), c->dims[t]) - c->cls_dim.begin());
  c->max_dim = c->cls_dim.back();
  const bool part = (cfg->flags & FLECHE_FLAG_STATIC_PER_TABLE) != 0;
  const bool bytes = c->cls_dim.size() > 1 && !part;
  c->per_table_launch = (cfg->flags & FLECHE_FLAG_PER_TABLE_LAUNCH) != 0;
  if (c->key_bits < 0) {
    delete c;
    return FLECHE_EINVAL;
  }
  auto fail = [&](fleche_status s) {
    free_all(c);
    delete c;
    return s;
  };
  if (cudaSetDevice(c->device) != cudaSuccess) return fail(FLECHE_EINVAL);
  cudaDeviceGetAttribute(&c->sm_count, cudaDevAttrMultiProcessorCount, c->device);

  Dev& dv = c->dv;
  uint64_t sets, rows = 0;
  size_t slab_bytes;
  std::vector<uint32_t> p_off(n, 0), p_sets(n, 0), p_rows(n, 0);
  std::vector<int64_t> p_slab(n, 0);
  if (part) {  // static per-table partitions: rows_t = floor(frac * c_t), frac = cache / table bytes
    unsigned __int128 tot = 0;
    for (int t = 0; t < n; ++t) tot += (unsigned __int128)c->card[t] * (uint64_t)c->dims[t] * 4u;
    uint64_t set_acc = 0, floats = 0;
    c->capacity_bytes = 0;
    for (int t = 0; t < n; ++t) {
      const uint64_t r = (uint64_t)(((unsigned __int128)cfg->cache_bytes * (uint64_t)c->card[t]) / tot);
      p_rows[t] = (uint32_t)std::min<uint64_t>(r, 0xFFFFFFE0ull);
      p_sets[t] = (p_rows[t] + 31) / 32;
      p_off[t] = (uint32_t)set_acc;
      p_slab[t] = (int64_t)floats;
      set_acc += p_sets[t];
      floats += (uint64_t)p_sets[t] * 32u * (uint64_t)c->dims[t];
      c->capacity_bytes += (uint64_t)p_rows[t] * 4u * (uint64_t)c->dims[t];
    }
    if (set_acc + 1 > 0xFFFFFFF0ull / 32) return fail(FLECHE_EINVAL);
    sets = set_acc + 1;  // + one padding set (a 0-row partition points past the last one)
    slab_bytes = (size_t)floats * 4u;
  } else if (!bytes) {  // uniform layout: way w of set s = slab row 32s + w
    rows = cfg->cache_bytes / (4ull * (uint64_t)c->max_dim);
    if (rows > 0xFFFFFFE0ull) return fail(FLECHE_EINVAL);
    sets = std::max<uint64_t>(1, (rows + 31) / 32);
    slab_bytes = (size_t)sets * 32u * (size_t)c->max_dim * 4u;
    c->capacity_bytes = rows * 4ull * (uint64_t)c->max_dim;
  } else {       // bytes layout: every set owns a set_bytes region (R22)
    uint64_t set_bytes = 4096;
    if (const char* e = getenv("FLECHE_SET_BYTES")) set_bytes = strtoull(e, nullptr, 10);
    if (set_bytes < 1024 || set_bytes > 4096 || (set_bytes & 31)) return fail(FLECHE_EINVAL);
    sets = cfg->cache_bytes / set_bytes;
    dv.set_units = sets ? (uint32_t)(set_bytes / 32) : 0u;  // a budget below one set caches nothing
    sets = std::max<uint64_t>(1, sets);
    if (sets > 0xFFFFFFF0ull / 32) return fail(FLECHE_EINVAL);
    slab_bytes = (size_t)sets * set_bytes;
    c->capacity_bytes = dv.set_units ? sets * set_bytes : 0;
  }
  const uint32_t scr_n = next_pow2(std::max<uint64_t>(1024, 2ull * (uint64_t)cfg->max_lookups));
  c->slab_floats = slab_bytes / 4;
  dv.bytes = bytes ? 1 : 0;
  dv.part = part ? 1 : 0;
  dv.sets = (uint32_t)sets;
  dv.rows = (uint32_t)rows;
  dv.dim = c->max_dim;
  dv.hash_seed = cfg->hash_seed;
  dv.scr_mask = scr_n - 1;
  const double p = cfg->admit_prob;
  dv.admit_all = (p <= 0.0 || p >= 1.0) ? 1 : 0;
  dv.admit_thr = dv.admit_all ? ~0ull : (uint64_t)ldexp(p, 64);
  dv.admit_seed = cfg->admit_seed;
  if (const char* e = getenv("FLECHE_KM_BLOCKS_PER_SM")) c->km_bps = std::max(1, atoi(e));
#ifdef FLECHE_EXPERIMENTS
  if (const char* e = getenv("FLECHE_EXP_MODE")) dv.exp_mode = atoi(e);
#endif

  auto alloc = [&](void** ptr, size_t b) { return cudaMalloc(ptr, std::max<size_t>(b, 16)) == cudaSuccess; };
  const size_t ways = (size_t)sets * 32u;
  bool ok = alloc((void**)&dv.keys, ways * 4) && alloc((void**)&dv.ts, ways * 4) && alloc((void**)&dv.slab, slab_bytes) &&
            alloc((void**)&dv.scratch, (size_t)scr_n * 8) && alloc((void**)&dv.owner_off, (size_t)scr_n * 8) &&
            alloc((void**)&dv.miss, (size_t)cfg->max_lookups * sizeof(MissRec)) &&
            alloc((void**)&dv.dup, (size_t)cfg->max_lookups * sizeof(DupRec)) && alloc((void**)&dv.ctl, sizeof(Ctl)) &&
            alloc((void**)&dv.stats, sizeof(unsigned long long) * kStripes * kNumCtr) &&
            alloc((void**)&c->d_tables, sizeof(TableInfo) * n);
  if (ok) ok = alloc((void**)&dv.firstpos, (size_t)scr_n * 8);
  if (ok && bytes) ok = alloc((void**)&dv.loc, ways * 2) && alloc((void**)&dv.lock, (size_t)sets * 4);
  if (ok && !bytes) ok = alloc((void**)&dv.ipos, ways * 8);
  if (!ok) {
    cudaGetLastError();
    return fail(FLECHE_ENOMEM);
  }
  c->index_bytes = ways * (bytes ? 10 : 16) + (bytes ? (size_t)sets * 4 : 0) + (size_t)scr_n * 24 +
                   (size_t)cfg->max_lookups * (sizeof(MissRec) + sizeof(DupRec));
  dv.tables = c->d_tables;
  {  // flat key -> table decoding table (prefix match of the size-aware code), for key-sharded queries
    std::vector<uint64_t> kd(n);
    for (int t = 0; t < n; ++t) kd[t] = (c->base[t] << 16) | (uint64_t)t;
    std::sort(kd.begin(), kd.end());
    if (!alloc((void**)&c->d_kdec, 8ull * n) || cudaMemcpy(c->d_kdec, kd.data(), 8ull * n, cudaMemcpyHostToDevice) != cudaSuccess)
      return fail(FLECHE_ENOMEM);
    dv.kdec = c->d_kdec;
    dv.ntables = n;
  }
  if (cudaMemset(dv.keys, 0xFF, ways * 4) != cudaSuccess || cudaMemset(dv.ts, 0, ways * 4) != cudaSuccess ||
      cudaMemset(dv.scratch, 0, (size_t)scr_n * 8) != cudaSuccess ||
      cudaMemset(dv.stats, 0, sizeof(unsigned long long) * kStripes * kNumCtr) != cudaSuccess)
    return fail(FLECHE_ECUDA);
  if (bytes && (cudaMemset(dv.loc, 0, ways * 2) != cudaSuccess || cudaMemset(dv.lock, 0, (size_t)sets * 4) != cudaSuccess))
    return fail(FLECHE_ECUDA);
  if (!bytes && cudaMemset(dv.ipos, 0, ways * 8) != cudaSuccess) return fail(FLECHE_ECUDA);
  if (cudaMemset(dv.firstpos, 0xFF, (size_t)scr_n * 8) != cudaSuccess) return fail(FLECHE_ECUDA);
  Ctl ctl{};
  ctl.epoch = 1;
  ctl.ha_frac_q16 = 0;  // set below once the host-assisted fetch is configured
  if (cudaMemcpy(dv.ctl, &ctl, sizeof(Ctl), cudaMemcpyHostToDevice) != cudaSuccess) return fail(FLECHE_ECUDA);

  std::vector<const float*> dptr;
  if (register_host(c, cfg->host_tables, dptr) != FLECHE_OK) return fail(FLECHE_ECUDA);
  std::vector<TableInfo> ti(n);
  for (int t = 0; t < n; ++t)
    ti[t] = TableInfo{dptr[t], c->card[t], (uint32_t)c->base[t], c->dims[t], c->cls[t], p_off[t], p_sets[t],
                      p_rows[t], p_slab[t], c->hashed[t] ? (uint32_t)((1ull << c->fbits[t]) - 1) : 0u,
                      c->hashed[t]};
  if (cudaMemcpy(c->d_tables, ti.data(), sizeof(TableInfo) * n, cudaMemcpyHostToDevice) != cudaSuccess)
    return fail(FLECHE_ECUDA);
  {  // address-ordered miss scratch (uniform layout): slot0 monotone in the host-row address
    uint64_t lo = ~0ull, hi = 0;
    for (int t = 0; t < n; ++t) {
      lo = std::min<uint64_t>(lo, (uint64_t)dptr[t]);
      hi = std::max<uint64_t>(hi, (uint64_t)dptr[t] + (uint64_t)c->card[t] * (uint64_t)c->dims[t] * 4u);
    }
    const uint64_t span = hi - lo;
    // only worth it when the host tier outgrows the host link's translation reach (~1 GiB
    // measured, profiles/hostlink_locality_r01.json); below that the scan costs more than it saves
    uint64_t min_span = 1ull << 30;
    if (const char* e = getenv("FLECHE_ORDER_MIN_SPAN")) min_span = strtoull(e, nullptr, 10);
    dv.ordered = (!bytes && !part && span > (uint64_t)scr_n && span >= min_span && getenv("FLECHE_NO_ORDER") == nullptr)
                     ? 1 : 0;
    dv.bands = getenv("FLECHE_KM_BANDS") ? atoi(getenv("FLECHE_KM_BANDS")) : 2;  // 1-2 measured best at cfg2, 8 at cfg5 (profiles/km_bands_r02.txt)
    dv.host_lo = lo;
    dv.host_mul = dv.ordered ? (uint64_t)(((unsigned __int128)scr_n << 64) / span) : 0;
  }
  if (cudaEventCreateWithFlags(&c->chain_ev, cudaEventDisableTiming) != cudaSuccess) return fail(FLECHE_ECUDA);
  // KM: enough warps for the expected unique misses, km_bps CTAs of 4 warps per SM, and no
  // more CTAs than fit at once (cooperative launch: its grid barrier needs them all resident)
  // host-assisted miss fetch: forced by the flag, else by default on a large host tier
  // (the translation-bound regime of scattered zero-copy reads): cfg2 +25-33 %, cfg5 +45 %,
  // cfg4 (mixed widths) +27 % over zero-copy (profiles/bench_r02_*)
  uint64_t tier_bytes = 0;
  for (int t = 0; t < n; ++t) tier_bytes += (uint64_t)c->card[t] * (uint64_t)c->dims[t] * 4u;
  const unsigned ncpu = std::thread::hardware_concurrency();
  const bool use_ha = (cfg->flags & FLECHE_FLAG_HOST_ASSIST) ||
                      (!(cfg->flags & FLECHE_FLAG_NO_HOST_ASSIST) && !part && !c->per_table_launch &&
                       tier_bytes >= (1ull << 30) && ncpu >= 8 && !(getenv("FLECHE_HA") && !atoi(getenv("FLECHE_HA"))));
  c->km_smem = (size_t)kKmWarps * ((bytes ? kKmSmemF4 : 0) + (use_ha ? kHaSmemF4 : 0)) * sizeof(float4);
  {
    const void* km = (const void*)km_fn(bytes, c->cls_dim.size() == 1 ? c->max_dim : 0);
    if (c->km_smem > 48 * 1024 &&
        cudaFuncSetAttribute(km, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)c->km_smem) != cudaSuccess)
      return fail(FLECHE_ECUDA);
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, km, 128, c->km_smem) != cudaSuccess || per_sm < 1)
      return fail(FLECHE_ECUDA);
    c->km_blocks = (int)std::min<int64_t>((int64_t)std::min(c->km_bps, per_sm) * c->sm_count,
                                          std::max<int64_t>(1, (cfg->max_lookups + 255) / 256));
  }
  {  // KQ hit gather through the TMA engine (FLECHE_KQ_TMA=0/1; uniform rows of 32 or 64 floats)
    const char* e = getenv("FLECHE_KQ_TMA");
    const bool want = e ? atoi(e) != 0 : false;
    if (want && !bytes && c->cls_dim.size() == 1 && (c->max_dim == 32 || c->max_dim == 64)) {
      c->kq_tma = c->max_dim;
      c->kq_smem = (size_t)4 * 32 * c->max_dim * sizeof(float);
    }
  }
  // decoupled hit copy: uniform layout only (the bytes layout compacts set regions in KM,
  // which may move rows a concurrent copy reads; epoch protection covers the uniform slots)
  c->decoupled = !bytes && !(cfg->flags & FLECHE_FLAG_FUSED_HIT_COPY) && getenv("FLECHE_FUSED_GATHER") == nullptr;
  if (const char* e = getenv("FLECHE_DECOUPLE_MIN")) c->decouple_min = strtoll(e, nullptr, 10);
  if (c->decoupled) {
    if (cudaStreamCreateWithFlags(&c->side, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->fork_ev, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->join_ev, cudaEventDisableTiming) != cudaSuccess ||
        cudaMalloc((void**)&c->d_slots, (size_t)cfg->max_lookups * 4) != cudaSuccess)
      return fail(FLECHE_ENOMEM);
  }
  if (use_ha) {
    HostAssist* h = c->ha = new (std::nothrow) HostAssist();
    if (!h) return fail(FLECHE_ENOMEM);
    auto env_u = [](const char* k, uint64_t dflt) {
      const char* e = getenv(k);
      return e ? strtoull(e, nullptr, 10) : dflt;
    };
    h->nthreads = (int)std::max<uint64_t>(
        1, std::min<uint64_t>(kHaMaxThreads, env_u("FLECHE_HA_THREADS", std::max(1u, std::min(12u, ncpu > 4 ? ncpu - 4 : 1)))));
    // staging: rows of the widest width, shared equally by the width classes (whole blocks
    // each); requests are indexed by staging row.  Default 128 MiB per epoch parity for one
    // width, 512 MiB for several (cfg4 stages ~470K misses per batch)
    const uint32_t ncls = (uint32_t)c->cls_dim.size();
    h->stage_floats = std::max<uint64_t>(1024, env_u("FLECHE_HA_STAGE_KB", ncls > 1 ? 524288 : 131072) << 8);
    {
      const uint64_t rows = std::min<uint64_t>(h->stage_floats / (uint64_t)c->max_dim,
                                               (uint64_t)cfg->max_lookups + kHaBlock * ncls);
      const uint64_t per = (rows / ncls) / kHaBlock * kHaBlock;
      for (uint32_t k = 0; k < 8; ++k) {
        h->rbase[k] = k < ncls ? (uint32_t)(k * per) : 0u;
        h->rcap[k] = k < ncls ? (uint32_t)per : 0u;
      }
      h->req_cap = (uint32_t)(per * ncls);
      h->stage_floats = (uint64_t)h->req_cap * (uint64_t)c->max_dim;
    }
    h->blk_cap = h->req_cap / kHaBlock + 2;
    const size_t o_req = 0, o_desc = o_req + 2 * sizeof(HaReq) * (size_t)h->req_cap, o_bell = o_desc + 2 * sizeof(HaDesc),
                 o_start = (o_bell + 8 + 63) & ~size_t(63), o_ready = (o_start + 8 + 127) & ~size_t(127), o_stage = (o_ready + 8ull * h->blk_cap + 255) & ~size_t(255),
                 total = o_stage + 2 * 4 * h->stage_floats;
    if (cudaHostAlloc(&h->mem, total, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) {
      cudaGetLastError();
      h->mem = nullptr;
      return fail(FLECHE_ENOMEM);
    }
    memset(h->mem, 0, o_stage);
    char* b = (char*)h->mem;
    h->req = (HaReq*)(b + o_req);
    h->desc = (HaDesc*)(b + o_desc);
    h->bell = (unsigned long long*)(b + o_bell);
    h->start = (unsigned long long*)(b + o_start);
    h->ready = (uint32_t*)(b + o_ready);
    h->stage = (float*)(b + o_stage);
    void* dmem = nullptr;
    if (cudaHostGetDevicePointer(&dmem, h->mem, 0) != cudaSuccess) return fail(FLECHE_ECUDA);
    char* db = (char*)dmem;
    dv.ha = 1;
    dv.ha_req = (HaReq*)(db + o_req);
    dv.ha_desc = (HaDesc*)(db + o_desc);
    dv.ha_bell = (unsigned long long*)(db + o_bell);
    dv.ha_start = (unsigned long long*)(db + o_start);
    dv.ha_ready = (uint32_t*)(db + o_ready);
    dv.ha_blk_cap = h->blk_cap;
    dv.ha_row_floats = (uint32_t)c->max_dim;
    for (int k = 0; k < 8; ++k) {
      dv.ha_rbase[k] = h->rbase[k];
      dv.ha_rcap[k] = h->rcap[k];
    }
    if (cudaMalloc((void**)&dv.ha_seen, 4ull * h->blk_cap) != cudaSuccess ||
        cudaMemset(dv.ha_seen, 0, 4ull * h->blk_cap) != cudaSuccess)
      return fail(FLECHE_ENOMEM);
    // early fetch (FLECHE_HA_EARLY=0 turns it off): KQ's first kf_ctas CTAs move staged
    // blocks into an HBM copy while the lookups run
    // request forwarding (FLECHE_HA_FWD = CTAs, 0 = KQ's lanes write the host list directly)
    c->fwd_ctas = (int)std::min<uint64_t>(64, env_u("FLECHE_HA_FWD", 8));
    if (c->fwd_ctas && (cudaMalloc((void**)&dv.ha_reqd, sizeof(HaReq) * (size_t)h->req_cap) != cudaSuccess ||
                        cudaMemset(dv.ha_reqd, 0, sizeof(HaReq) * (size_t)h->req_cap) != cudaSuccess))
      return fail(FLECHE_ENOMEM);
    c->kf_ctas = (int)env_u("FLECHE_HA_EARLY", 1) ? (int)std::min<uint64_t>(64, std::max<uint64_t>(1, env_u("FLECHE_KF_CTAS", 16))) : 0;
    dv.ha_kf_tail = (uint32_t)env_u("FLECHE_KF_TAIL", 0);
    c->kf_min = (int64_t)env_u("FLECHE_HA_EARLY_MIN", 524288);
    if (c->kf_ctas) {
      if (cudaMalloc((void**)&dv.ha_hstage, 2ull * 4ull * h->stage_floats) != cudaSuccess ||
          cudaMalloc((void**)&dv.ha_hseen, 4ull * h->blk_cap) != cudaSuccess ||
          cudaMemset(dv.ha_hseen, 0, 4ull * h->blk_cap) != cudaSuccess)
        return fail(FLECHE_ENOMEM);
    }
    dv.ha_stage = (float*)(db + o_stage);
    dv.ha_req_cap = h->req_cap;
    dv.ha_stage_floats = h->stage_floats;
    dv.ha_timeout_ns = env_u("FLECHE_HA_TIMEOUT_US", 2000) * 1000ull;
    {  // share of the staging blocks the host threads gather (the rest: KM's zero-copy reads)
      // (fixed shares measured: best 0.7-0.8 at 8.6 GB, cfg2 and cfg5, profiles/bench_r02_ha_*.json;
      // >= 0.85 at 113 GB, cfg3h, round 1)
      const char* e = getenv("FLECHE_HA_FRAC");
      // FLECHE_HA_FRAC fixes the share; otherwise the unified-index tuning loop (ui_tune,
      // P:L861-872) starts with the host threads taking every block and moves it by itself
      const double f = e ? std::min(1.0, std::max(0.0, atof(e))) : 1.0;
      const uint32_t frac_q16 = (uint32_t)(f * 65536.0 + 0.5);
      dv.ha_frac_fixed = e ? 1u : 0u;
      if (cudaMemcpy(&dv.ctl->ha_frac_q16, &frac_q16, 4, cudaMemcpyHostToDevice) != cudaSuccess)
        return fail(FLECHE_ECUDA);
      dv.ha_min_rows = (uint32_t)env_u("FLECHE_HA_MIN_ROWS", 1024);
      dv.ha_unit_pieces = (uint32_t)env_u("FLECHE_HA_UNIT_PIECES", 0);  // 0: adaptive (km_ha)
    }
    h->nt_stores = env_u("FLECHE_HA_NT", 1) != 0 && __builtin_cpu_supports("avx2");
    h->delay_ns = env_u("FLECHE_HA_DELAY_US", 0) * 1000ull;
    h->stream = env_u("FLECHE_HA_STREAM", 1) != 0;
    h->host.assign(cfg->host_tables, cfg->host_tables + n);
    h->card = c->card;
    h->dims = c->dims;
    for (int i = 0; i < h->nthreads; ++i) h->th.emplace_back(ha_worker, h, i);
  }
#ifdef FLECHE_EXPERIMENTS
  // KM warps x 4, then [exp_slots + 0..7] KQ stamps, [exp_slots + 8 + w] early-fetch warp w's exit,
  // [exp_slots + 264 + (epoch % 64) * 4 + {0,1,2}] per-batch ring: KQ start, lookups end, last fetch exit
  if (cudaMalloc((void**)&dv.exp_buf, ((size_t)c->km_blocks * 4 * 4 + 8 + 512) * 8) != cudaSuccess) return fail(FLECHE_ENOMEM);
  cudaMemset(dv.exp_buf, 0, ((size_t)c->km_blocks * 4 * 4 + 8 + 512) * 8);
  dv.exp_slots = (uint32_t)c->km_blocks * 16;
  if (c->ha) {
    if (cudaMalloc((void**)&dv.exp_blk, ((size_t)c->ha->blk_cap * 8) * 8) != cudaSuccess) return fail(FLECHE_ENOMEM);
    cudaMemset(dv.exp_blk, 0, ((size_t)c->ha->blk_cap * 8) * 8);
    c->ha->exp_pub = new uint64_t[c->ha->blk_cap]();
  }
#endif
  if (cudaDeviceSynchronize() != cudaSuccess) return fail(FLECHE_ECUDA);
  *out = c;
  return FLECHE_OK;
}

fleche_status fleche_query(fleche_ctx* c, const int64_t* const* ids, const int64_t* lengths, float* out,
                           fleche_stream stream) {
  if (!c || !ids || !lengths) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  return query_impl(c, ids, lengths, out, (cudaStream_t)stream);
}

fleche_status fleche_prefill(fleche_ctx* c, const int64_t* const* ids, const int64_t* lengths, fleche_stream stream) {
  if (!c || !ids || !lengths) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  int64_t floats = 0;
  for (int t = 0; t < c->n; ++t) {
    if (lengths[t] < 0) return FLECHE_EINVAL;
    floats += lengths[t] * (int64_t)c->dims[t];
  }
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  if (floats > c->prefill_floats) {  // the batch's rows land in a ctx-owned scratch output
    if (c->have_last) FL_CUDA(c, cudaStreamSynchronize(c->last_stream));
    if (c->d_prefill_out) FL_CUDA(c, cudaFree(c->d_prefill_out));
    c->d_prefill_out = nullptr;
    FL_CUDA(c, cudaMalloc((void**)&c->d_prefill_out, (size_t)floats * 4));
    c->prefill_floats = floats;
  }
  return query_impl(c, ids, lengths, c->d_prefill_out, (cudaStream_t)stream);
}

fleche_status fleche_query_pooled(fleche_ctx* c, const int64_t* const* ids, const int64_t* const* offsets,
                                  const int64_t* bags, const int64_t* nnz, float* out, fleche_stream stream) {
  if (!c || !ids || !offsets || !bags || !nnz) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  int64_t total_bags = 0;
  for (int t = 0; t < c->n; ++t) {
    if (bags[t] < 0 || nnz[t] < 0 || (bags[t] > 0 && !offsets[t])) return FLECHE_EINVAL;
    total_bags += bags[t];
  }
  if (total_bags > 0 && (!out || ((uintptr_t)out & 15u))) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  if (!c->d_pool_stage) FL_CUDA(c, cudaMalloc((void**)&c->d_pool_stage, (size_t)c->max_lookups * c->max_dim * 4));
  cudaStream_t s = (cudaStream_t)stream;
  // one-hot lookups of every ID into the staging rows (A1-A8), then bag sums (KP)
  st = query_impl(c, ids, nnz, c->d_pool_stage, s, 5);
  if (st != FLECHE_OK) return st;
  if (c->n <= 32) return launch_pool<32>(c, offsets, bags, nnz, out, s);
  if (c->n <= 128) return launch_pool<128>(c, offsets, bags, nnz, out, s);
  return launch_pool<FLECHE_MAX_TABLES>(c, offsets, bags, nnz, out, s);
}

fleche_status fleche_query_host(fleche_ctx* c, const int64_t* const* ids, const int64_t* lengths, float* out,
                                fleche_stream stream) {
  if (!c || !ids || !lengths) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  int64_t total = 0, out_floats = 0;
  for (int t = 0; t < c->n; ++t) {
    if (lengths[t] < 0 || (lengths[t] > 0 && !ids[t])) return FLECHE_EINVAL;
    total += lengths[t];
    out_floats += lengths[t] * (int64_t)c->dims[t];
  }
  if (total > c->max_lookups || (total > 0 && !out)) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  // Pipelined across calls: the lookups run on the ctx's host-call stream hq, the output
  // copy on a second stream hd from one of two staging buffers, so call k's device->host
  // copy overlaps call k+1's H2D + query; the caller's stream waits for this call's copy
  // (out is complete once it is synchronised).
  const cudaStream_t caller = (cudaStream_t)stream;
  if (!c->d_ids_stage) {
    FL_CUDA(c, cudaMalloc((void**)&c->d_ids_stage, (size_t)c->max_lookups * 8));
    FL_CUDA(c, cudaMalloc((void**)&c->d_out_stage, (size_t)c->max_lookups * (size_t)c->max_dim * 4));
    FL_CUDA(c, cudaMalloc((void**)&c->d_out_stage2, (size_t)c->max_lookups * (size_t)c->max_dim * 4));
    FL_CUDA(c, cudaStreamCreateWithFlags(&c->hq, cudaStreamNonBlocking));
    FL_CUDA(c, cudaStreamCreateWithFlags(&c->hd, cudaStreamNonBlocking));
    for (int i = 0; i < 2; ++i) {
      FL_CUDA(c, cudaEventCreateWithFlags(&c->hq_ev[i], cudaEventDisableTiming));
      FL_CUDA(c, cudaEventCreateWithFlags(&c->hd_ev[i], cudaEventDisableTiming));
      FL_CUDA(c, cudaEventCreateWithFlags(&c->hc_ev[i], cudaEventDisableTiming));
      FL_CUDA(c, cudaEventRecord(c->hd_ev[i], c->hd));
    }
  }
  const int par = c->hpar;
  c->hpar ^= 1;
  float* stage = par ? c->d_out_stage2 : c->d_out_stage;
  const cudaStream_t s = c->hq;
  // The lookups wait for the copy that last read this staging buffer (and, via order_on,
  // for the ctx's previous batch) but NOT for `stream`: `stream` already waits for the
  // previous call's output copy, so ordering the lookups after it would run copy k and
  // lookups k+1 one after the other.  The host IDs must therefore be final when the call is
  // made (header).  Measured on one B200 box, 8-9 alternating runs each: e2e 184-197
  // Mkeys/s overlapped (one outlier at 65) vs 98-174 ordered (profiles/e2e_overlap_ab_r01).
  // FLECHE_HOST_ORDERED=1 restores the strict order.  The output copy below always orders
  // after `stream`'s work (e.g. the caller's pending reads of out).
  FL_CUDA(c, cudaStreamWaitEvent(s, c->hd_ev[par], 0));
  FL_CUDA(c, cudaEventRecord(c->hc_ev[par], caller));
  static const bool ordered = getenv("FLECHE_HOST_ORDERED") != nullptr;
  if (ordered) FL_CUDA(c, cudaStreamWaitEvent(s, c->hc_ev[par], 0));
  st = order_on(c, s);
  if (st != FLECHE_OK) return st;
  std::vector<const int64_t*> dids(c->n);
  // one copy when the non-empty per-table host arrays are consecutive in memory, else one
  // per table (empty tables are skipped: their pointers may be anything)
  bool contiguous = true;
  const int64_t* expect = nullptr;
  for (int t = 0; t < c->n; ++t) {
    if (lengths[t] == 0) continue;
    if (expect && ids[t] != expect) contiguous = false;
    expect = ids[t] + lengths[t];
  }
  int64_t acc = 0;
  const int64_t* first = nullptr;
  for (int t = 0; t < c->n; ++t) {
    if (!first && lengths[t] > 0) first = ids[t];
    dids[t] = c->d_ids_stage + acc;
    if (!contiguous && lengths[t] > 0)
      FL_CUDA(c, cudaMemcpyAsync(c->d_ids_stage + acc, ids[t], (size_t)lengths[t] * 8, cudaMemcpyHostToDevice, s));
    acc += lengths[t];
  }
  if (contiguous && total > 0)
    FL_CUDA(c, cudaMemcpyAsync(c->d_ids_stage, first, (size_t)total * 8, cudaMemcpyHostToDevice, s));
  st = query_impl(c, dids.data(), lengths, stage, s);
  if (st != FLECHE_OK) return st;
  FL_CUDA(c, cudaEventRecord(c->hq_ev[par], s));
  FL_CUDA(c, cudaStreamWaitEvent(c->hd, c->hq_ev[par], 0));
  FL_CUDA(c, cudaStreamWaitEvent(c->hd, c->hc_ev[par], 0));  // whatever `stream` held (e.g. reads of out)
  if (out_floats > 0)
    FL_CUDA(c, cudaMemcpyAsync(out, stage, (size_t)out_floats * 4, cudaMemcpyDeviceToHost, c->hd));
  FL_CUDA(c, cudaEventRecord(c->hd_ev[par], c->hd));
  FL_CUDA(c, cudaStreamWaitEvent(caller, c->hd_ev[par], 0));
  return FLECHE_OK;
}

fleche_status fleche_stats(fleche_ctx* c, fleche_stats_t* out) {
  if (!c || !out) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  if (c->have_last) FL_CUDA(c, cudaStreamSynchronize(c->last_stream));
  std::vector<unsigned long long> h(kStripes * kNumCtr);
  Ctl ctl;
  FL_CUDA(c, cudaMemcpy(h.data(), c->dv.stats, h.size() * 8, cudaMemcpyDeviceToHost));
  FL_CUDA(c, cudaMemcpy(&ctl, c->dv.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost));
  unsigned long long v[kNumCtr] = {0};
  for (int s = 0; s < kStripes; ++s)
    for (int k = 0; k < kNumCtr; ++k) v[k] += h[s * kNumCtr + k];
  memset(out, 0, sizeof(*out));
  out->batches = c->batches;
  out->lookups = c->lookups;
  out->hits = v[C_HITS];
  out->misses = v[C_MISSES];
  out->invalid = v[C_INVALID];
  out->unique_hits = v[C_UHITS];
  out->unique_misses = v[C_UMISS];
  out->unique_keys = v[C_UHITS] + v[C_UMISS];
  out->inserted = v[C_INSERTED];
  out->evicted = v[C_EVICTED];
  out->bypassed = v[C_BYPASSED];
  out->occupancy_bytes = (uint64_t)ctl.occ_bytes;
  out->capacity_bytes = c->capacity_bytes;
  out->index_bytes = c->index_bytes;
  out->host_bytes_fetched = v[C_HOSTBYTES];
  out->kernels_launched = c->kernels;
  out->assisted_rows = v[C_HAROWS];
  out->assist_timeouts = v[C_HATIMEOUT];
  out->scans = v[C_SCANS];
  out->ui_share_ppm = c->ha ? (uint64_t)(65536u - std::min(65536u, ctl.ha_frac_q16)) * 1000000ull / 65536ull : 0;
  return ctl.err_invalid ? FLECHE_ERANGE : FLECHE_OK;
}

fleche_status fleche_reset_stats(fleche_ctx* c) {
  if (!c) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  if (c->have_last) FL_CUDA(c, cudaStreamSynchronize(c->last_stream));
  FL_CUDA(c, cudaMemset(c->dv.stats, 0, sizeof(unsigned long long) * kStripes * kNumCtr));
  FL_CUDA(c, cudaMemset(&c->dv.ctl->err_invalid, 0, sizeof(uint32_t)));
  FL_CUDA(c, cudaDeviceSynchronize());
  c->batches = c->lookups = c->kernels = 0;
  return FLECHE_OK;
}

fleche_status fleche_destroy(fleche_ctx* c) {
  if (!c) return FLECHE_EINVAL;
  int cur = -1;
  cudaGetDevice(&cur);
  if (cur != c->device) cudaSetDevice(c->device);
  if (c->have_last) cudaStreamSynchronize(c->last_stream);
  if (c->hd) cudaStreamSynchronize(c->hd);  // fleche_query_host's last output copy
  free_all(c);
  delete c;
  return FLECHE_OK;
}

fleche_status fleche_get_encoding(fleche_ctx* c, uint64_t* base, int32_t* fbits, int32_t* key_bits) {
  if (!c) return FLECHE_EINVAL;
  for (int t = 0; t < c->n; ++t) {
    if (base) base[t] = c->base[t];
    if (fbits) fbits[t] = c->fbits[t];
  }
  if (key_bits) *key_bits = c->key_bits;
  return FLECHE_OK;
}

fleche_status fleche_encode(int32_t n, const int64_t* cards, int32_t key_bits, uint64_t* base, int32_t* fbits,
                            int32_t* hashed, int32_t* key_bits_out) {
  if (n < 1 || n > FLECHE_MAX_TABLES || !cards || !base || !fbits || !key_bits_out || key_bits < 0 || key_bits > 32)
    return FLECHE_EINVAL;
  std::vector<int64_t> card(cards, cards + n);
  for (int64_t c : card)
    if (c < 1) return FLECHE_EINVAL;
  std::vector<uint64_t> b;
  std::vector<int32_t> fb, h(n, 0);
  int kb = size_aware_code(card, b, fb);  // same steps as fleche_create
  if (key_bits > 0 && (kb < 0 || key_bits < kb)) {
    if (short_code(card, key_bits, b, fb, h) < 0) return FLECHE_EINVAL;
    kb = key_bits;
  }
  if (kb < 0) return FLECHE_EINVAL;
  for (int t = 0; t < n; ++t) {
    base[t] = b[t];
    fbits[t] = fb[t];
    if (hashed) hashed[t] = h[t];
  }
  *key_bits_out = kb;
  return FLECHE_OK;
}

fleche_status fleche_get_geometry(fleche_ctx* c, int64_t* sets, int64_t* rows, int32_t* row_floats) {
  if (!c) return FLECHE_EINVAL;
  if (sets) *sets = c->dv.sets;
  if (rows) *rows = (c->dv.bytes || c->dv.part) ? 0 : c->dv.rows;
  if (row_floats) *row_floats = c->dv.part ? 0 : (c->dv.bytes ? -(int32_t)(c->dv.set_units * 8) : c->max_dim);
  return FLECHE_OK;
}

fleche_status fleche_debug_snapshot(fleche_ctx* c, uint32_t* keys, uint32_t* ts, size_t ways_cap, float* slab,
                                    size_t slab_floats_cap) {
  if (!c) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  const size_t ways = (size_t)c->dv.sets * 32u;
  const size_t slab_floats = c->slab_floats;
  if ((keys || ts) && ways_cap < ways) return FLECHE_EINVAL;
  if (slab && slab_floats_cap < slab_floats) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  if (c->have_last) FL_CUDA(c, cudaStreamSynchronize(c->last_stream));
  if (keys) FL_CUDA(c, cudaMemcpy(keys, c->dv.keys, ways * 4, cudaMemcpyDeviceToHost));
  if (ts) FL_CUDA(c, cudaMemcpy(ts, c->dv.ts, ways * 4, cudaMemcpyDeviceToHost));
  if (slab && slab_floats) FL_CUDA(c, cudaMemcpy(slab, c->dv.slab, slab_floats * 4, cudaMemcpyDeviceToHost));
  return FLECHE_OK;
}

fleche_status fleche_debug_locations(fleche_ctx* c, uint16_t* loc, size_t ways_cap) {
  if (!c || !loc) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  const size_t ways = (size_t)c->dv.sets * 32u;
  if (!c->dv.bytes || ways_cap < ways) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  if (c->have_last) FL_CUDA(c, cudaStreamSynchronize(c->last_stream));
  FL_CUDA(c, cudaMemcpy(loc, c->dv.loc, ways * 2, cudaMemcpyDeviceToHost));
  return FLECHE_OK;
}

// Diagnostics (tools only): copy the device control block to host on a private
// non-blocking stream, so it can be read while the ctx's own streams are stuck.
fleche_status fleche_debug_ctl(fleche_ctx* c, void* host, size_t bytes) {
  if (!c || !host || bytes < sizeof(Ctl)) return FLECHE_EINVAL;
  cudaStream_t t;
  if (cudaStreamCreateWithFlags(&t, cudaStreamNonBlocking) != cudaSuccess) return FLECHE_ECUDA;
  cudaMemcpyAsync(host, c->dv.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, t);
  const cudaError_t e = cudaStreamSynchronize(t);
  cudaStreamDestroy(t);
  return e == cudaSuccess ? FLECHE_OK : FLECHE_ECUDA;
}

fleche_status fleche_set_watermarks(fleche_ctx* c, double hi, double lo) {
  if (!c) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  if (!(hi > 0.0) || !(lo > 0.0) || lo > hi || c->dv.part) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  if (c->have_last) FL_CUDA(c, cudaStreamSynchronize(c->last_stream));
  if (hi >= 1.0) {  // never above capacity: the canonical on-demand policy
    c->wm_on = false;
    return FLECHE_OK;
  }
  if (!c->d_age_hist) {
    FL_CUDA(c, cudaMalloc((void**)&c->d_age_hist, kAgeBins * 8));
    FL_CUDA(c, cudaMemset(c->d_age_hist, 0, kAgeBins * 8));
    FL_CUDA(c, cudaDeviceSynchronize());
  }
  const double cap = (double)c->capacity_bytes;
  c->wm_hi = (long long)(hi * cap);
  c->wm_lo = (long long)(lo * cap);
  const int64_t quads = (int64_t)c->dv.sets * 8;
  c->ke_blocks = (int)std::max<int64_t>(1, std::min<int64_t>((quads + 255) / 256, (int64_t)c->sm_count * 4));
  c->wm_on = true;
  return FLECHE_OK;
}

fleche_status fleche_set_profiling(fleche_ctx* c, int enable) {
  if (!c) return FLECHE_EINVAL;
  c->profiling = enable != 0;
  return FLECHE_OK;
}

fleche_status fleche_kernel_times_ex(fleche_ctx* c, double* ms4, uint64_t* queries) {
  if (!c) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  double acc[4] = {0, 0, 0, 0};
  size_t i = 0;
  for (int k : c->ev_kinds) {  // events: [start, after KQ, after KM (incl. restore), same again (, after KP)]
    FL_CUDA(c, cudaEventSynchronize(c->ev_pool[i + k - 1]));
    for (int j = 0; j + 1 < k; ++j) {
      float x = 0;
      FL_CUDA(c, cudaEventElapsedTime(&x, c->ev_pool[i + j], c->ev_pool[i + j + 1]));
      acc[j] += x;
    }
    i += k;
  }
  if (ms4)
    for (int j = 0; j < 4; ++j) ms4[j] = acc[j];
  if (queries) *queries = c->ev_kinds.size();
  c->ev_used = 0;
  c->ev_kinds.clear();
  return FLECHE_OK;
}

fleche_status fleche_kernel_times(fleche_ctx* c, double* kq_ms, double* ki_ms, uint64_t* queries) {
  double ms4[4];
  fleche_status st = fleche_kernel_times_ex(c, ms4, queries);
  if (st != FLECHE_OK) return st;
  if (kq_ms) *kq_ms = ms4[0];
  if (ki_ms) *ki_ms = ms4[1] + ms4[2] + ms4[3];
  return FLECHE_OK;
}

fleche_status fleche_probe_host_read(const void* host, uint64_t bytes, int32_t row_bytes, int64_t rows, uint64_t seed,
                                     fleche_stream stream, double* gbps) {
  if (!host || !gbps || rows < 1 || row_bytes < 16 || (row_bytes & 15) || bytes < (uint64_t)row_bytes)
    return FLECHE_EINVAL;
  const int D = row_bytes / 4;
  if (D != 32 && D != 64 && D != 128 && D != 256) return FLECHE_EINVAL;
  void* dev = nullptr;
  if (cudaHostGetDevicePointer(&dev, (void*)host, 0) != cudaSuccess) return FLECHE_EINVAL;
  float* sink = nullptr;
  if (cudaMalloc((void**)&sink, 4096ull * row_bytes) != cudaSuccess) return FLECHE_ENOMEM;
  cudaStream_t s = (cudaStream_t)stream;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const uint64_t span = bytes / (uint64_t)row_bytes;
  const unsigned blocks = (unsigned)((rows + 127) / 128);
  auto launch = [&](uint64_t sd) {
    launch_k(kPdlNone, probe_fn(D), blocks, 128, 0, s, (const float*)dev, span, rows, sd, sink);
  };
  launch(seed * 0x9E3779B97F4A7C15ull + 0x632BE59BD9B4E019ull);  // warm-up (clocks), rows disjoint from the timed ones
  cudaEventRecord(e0, s);
  launch(seed);
  cudaEventRecord(e1, s);
  cudaError_t e = cudaEventSynchronize(e1);
  float ms = 0;
  if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFree(sink);
  if (e != cudaSuccess) return FLECHE_ECUDA;
  *gbps = (double)rows * (double)row_bytes / ((double)ms * 1e-3) / 1e9;
  return FLECHE_OK;
}

}  // extern "C"

// ---------------------------------------------------------------- key-sharded mode
namespace {

template <int MAXT>
fleche_status launch_keys(fleche_ctx* c, const uint32_t* keys, int64_t count, float* rows, uint8_t* flags,
                          cudaStream_t s, const uint32_t* const* segs = nullptr, const int64_t* seg_counts = nullptr,
                          int nseg = 0, const int64_t* dcnt = nullptr, int me = 0) {
  QArgs<MAXT> qa;
  memset(&qa, 0, sizeof(qa));  // out_off[t] = 0: row g of `rows` answers keys[g]
  qa.n = 1;
  qa.scan[1] = count;
  qa.out = rows;
  qa.fkeys = keys;
  qa.hit_flags = flags;
  if (segs) {  // segments in order: row g answers the g-th key of their concatenation
    qa.fkseg = 1;
    qa.n = nseg;
    int64_t acc = 0;
    for (int i = 0; i < nseg; ++i) {
      qa.ids[i] = (const int64_t*)segs[i];
      qa.scan[i] = acc;
      acc += seg_counts ? seg_counts[i] : 0;
    }
    qa.scan[nseg] = acc;
    qa.fkeys = segs[0];  // non-null: the flat-key path
    qa.dcnt = dcnt;      // sync-free: the counts are read on the device; the grid strides over them
    qa.dme = me;
  }
  KMArgs ka;
  memset(&ka, 0, sizeof(ka));
  ka.out = rows;
  ka.ncls = 1;
  ka.cls_dim[0] = c->max_dim;
  qa.ncls = 1;
  qa.ha_bell = c->dv.ha;  // host-assisted owner: KQ's last CTA rings the doorbell (as in launch_query)
  fleche_status st = prof_event(c, s, true, 4);
  if (st != FLECHE_OK) return st;
  if (dcnt) {  // count unknown on the host: a capacity-sized, grid-strided launch (TD = 0: no TMA variant)
    const int64_t blocks = std::min<int64_t>((c->max_lookups + FL_KQ_THREADS - 1) / FL_KQ_THREADS,
                                             (int64_t)FL_KQ_MIN_BLOCKS * c->sm_count);
    launch_k(kPdlKQ, kq_fn<MAXT>(0), (unsigned)std::max<int64_t>(1, blocks), FL_KQ_THREADS, 0, s, qa, c->dv);
    c->kernels++;
  } else if (count > 0) {
    launch_k(kPdlKQ, kq_fn<MAXT>(c->kq_tma), (unsigned)((count + FL_KQ_THREADS - 1) / FL_KQ_THREADS), FL_KQ_THREADS,
             c->kq_smem, s, qa, c->dv);
    c->kernels++;
  }
  if ((st = prof_event(c, s, false, 0)) != FLECHE_OK) return st;
  launch_miss(c, s, ka);
  if ((st = prof_event(c, s, false, 0)) != FLECHE_OK) return st;
  launch_scan(c, s);
  if ((st = prof_event(c, s, false, 0)) != FLECHE_OK) return st;
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return poison(c, e, "kernel launch");
  return FLECHE_OK;
}

template <int MAXT>
void fill_rargs(fleche_ctx* c, RArgs<MAXT>& ra, const int64_t* const* ids, const int64_t* lengths) {
  memset(&ra, 0, sizeof(ra));
  ra.n = c->n;
  ra.repoch = c->repoch;
  int64_t acc = 0, oacc = 0;
  for (int t = 0; t < c->n; ++t) {
    if (ids) ra.ids[t] = ids[t];
    ra.scan[t] = acc;
    ra.out_off[t] = oacc;
    acc += lengths[t];
    oacc += lengths[t] * (int64_t)c->dims[t];
  }
  ra.scan[c->n] = acc;
}

template <int MAXT>
fleche_status launch_route(fleche_ctx* c, const int64_t* const* ids, const int64_t* lengths, int64_t total,
                           uint32_t* send_keys, int64_t* send_counts, cudaStream_t s) {
  RArgs<MAXT> ra;
  fill_rargs<MAXT>(c, ra, ids, lengths);
  if (total > 0) {
    launch_k(kPdlNone, kr_fn<MAXT>(), (unsigned)((total + 127) / 128), 128, 0, s, ra, c->rd,
             (const TableInfo*)c->d_tables);
    c->kernels++;
  }
  launch_k(kPdlNone, kpk_fn(), (unsigned)std::max(1, std::min(2 * c->sm_count, (int)((total + 255) / 256))), 256, 0, s,
           c->rd, send_keys, send_counts, c->route_peer);
  c->kernels++;
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return poison(c, e, "kernel launch");
  return FLECHE_OK;
}

template <int MAXT, int D>
fleche_status launch_restore_d(fleche_ctx* c, const float* rows, const uint8_t* flags, float* out, cudaStream_t s,
                               const PeerArgs& pa) {
  RArgs<MAXT> ra;
  fill_rargs<MAXT>(c, ra, nullptr, c->route_len.data());
  const int64_t total = ra.scan[c->n];
  if (total > 0) {
    launch_k(kPdlNone, krs_fn<MAXT>(D), (unsigned)((total + 127) / 128), 128, 0, s, ra, c->rd, rows, flags, out, pa);
    c->kernels++;
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return poison(c, e, "kernel launch");
  return FLECHE_OK;
}

template <int MAXT>
fleche_status launch_restore(fleche_ctx* c, const float* rows, const uint8_t* flags, float* out, cudaStream_t s,
                             const PeerArgs& pa) {
  switch (c->max_dim) {
    case 8: return launch_restore_d<MAXT, 8>(c, rows, flags, out, s, pa);
    case 16: return launch_restore_d<MAXT, 16>(c, rows, flags, out, s, pa);
    case 32: return launch_restore_d<MAXT, 32>(c, rows, flags, out, s, pa);
    case 64: return launch_restore_d<MAXT, 64>(c, rows, flags, out, s, pa);
    case 128: return launch_restore_d<MAXT, 128>(c, rows, flags, out, s, pa);
    default: return launch_restore_d<MAXT, 256>(c, rows, flags, out, s, pa);
  }
}

bool uniform_dims(const fleche_ctx* c) { return c->cls_dim.size() == 1; }

}  // namespace

extern "C" {

fleche_status fleche_route(fleche_ctx* c, const int64_t* const* ids, const int64_t* lengths, int32_t world,
                           uint32_t owner_seed, uint32_t* send_keys, int64_t* send_counts, fleche_stream stream) {
  if (!c || !ids || !lengths || !send_keys || !send_counts || world < 1 || world > kMaxWorld) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  if (!uniform_dims(c) || c->lossy) return FLECHE_EINVAL;
  int64_t total = 0;
  for (int t = 0; t < c->n; ++t) {
    if (lengths[t] < 0 || (lengths[t] > 0 && !ids[t])) return FLECHE_EINVAL;
    total += lengths[t];
  }
  if (total > c->max_lookups) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  if (!c->rd_ready || c->rd.world != world) {
    if (c->rd_ready) FL_CUDA(c, cudaStreamSynchronize(c->last_stream));
    void* ptrs[] = {c->rd.scratch, c->rd.slotval, c->rd.inv, c->rd.region, c->rd.cnt, c->rd.prefix, c->rd.done,
                    c->rd.stats};
    for (void* p : ptrs)
      if (p) cudaFree(p);
    const uint32_t scr_n = next_pow2(std::max<uint64_t>(1024, 2ull * (uint64_t)c->max_lookups));
    RouteDev& rd = c->rd;
    rd = RouteDev{};
    rd.mask = scr_n - 1;
    rd.cap = (uint32_t)c->max_lookups;
    rd.world = world;
    rd.owner_seed = owner_seed;
    FL_CUDA(c, cudaMalloc((void**)&rd.scratch, (size_t)scr_n * 8));
    FL_CUDA(c, cudaMalloc((void**)&rd.slotval, (size_t)scr_n * 8));
    FL_CUDA(c, cudaMalloc((void**)&rd.inv, (size_t)c->max_lookups * 4));
    FL_CUDA(c, cudaMalloc((void**)&rd.region, (size_t)world * c->max_lookups * 4));
    FL_CUDA(c, cudaMalloc((void**)&rd.cnt, kMaxWorld * 4));
    FL_CUDA(c, cudaMalloc((void**)&rd.prefix, (kMaxWorld + 1) * 8));
    FL_CUDA(c, cudaMalloc((void**)&rd.done, 4));
    FL_CUDA(c, cudaMalloc((void**)&rd.stats, 4 * 8));
    FL_CUDA(c, cudaMemset(rd.scratch, 0, (size_t)scr_n * 8));
    FL_CUDA(c, cudaMemset(rd.cnt, 0, kMaxWorld * 4));
    FL_CUDA(c, cudaMemset(rd.done, 0, 4));
    FL_CUDA(c, cudaMemset(rd.stats, 0, 32));
    FL_CUDA(c, cudaDeviceSynchronize());
    c->rd_ready = true;
    c->repoch = 0;
  }
  c->rd.owner_seed = owner_seed;
  st = order_on(c, s);
  if (st != FLECHE_OK) return st;
  ++c->repoch;
  c->route_len.assign(lengths, lengths + c->n);
  if (c->n <= 32) return launch_route<32>(c, ids, lengths, total, send_keys, send_counts, s);
  if (c->n <= 128) return launch_route<128>(c, ids, lengths, total, send_keys, send_counts, s);
  return launch_route<FLECHE_MAX_TABLES>(c, ids, lengths, total, send_keys, send_counts, s);
}

fleche_status fleche_query_keys(fleche_ctx* c, const uint32_t* keys, int64_t count, float* rows, uint8_t* hit_flags,
                                fleche_stream stream) {
  if (!c || count < 0 || (count > 0 && (!keys || !rows))) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  if (!uniform_dims(c) || c->dv.part || count > c->max_lookups || ((uintptr_t)rows & 15u)) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  st = order_on(c, s);
  if (st != FLECHE_OK) return st;
  if (c->n <= 32) st = launch_keys<32>(c, keys, count, rows, hit_flags, s);
  else if (c->n <= 128) st = launch_keys<128>(c, keys, count, rows, hit_flags, s);
  else st = launch_keys<FLECHE_MAX_TABLES>(c, keys, count, rows, hit_flags, s);
  if (st == FLECHE_OK) {
    c->batches++;
    c->lookups += (uint64_t)count;
  }
  return st;
}

fleche_status fleche_query_keys_seg(fleche_ctx* c, const uint32_t* const* segs, const int64_t* counts, int32_t nseg,
                                    float* rows, uint8_t* hit_flags, fleche_stream stream) {
  if (!c || !segs || !counts || nseg < 1 || nseg > kMaxWorld || !rows || ((uintptr_t)rows & 15u)) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  int64_t count = 0;
  for (int i = 0; i < nseg; ++i) {
    if (counts[i] < 0 || (counts[i] > 0 && !segs[i])) return FLECHE_EINVAL;
    count += counts[i];
  }
  if (!uniform_dims(c) || c->dv.part || count > c->max_lookups) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  st = order_on(c, s);
  if (st != FLECHE_OK) return st;
  std::vector<const uint32_t*> sg(segs, segs + nseg);
  for (auto& p : sg)
    if (!p) p = segs[0] ? segs[0] : reinterpret_cast<const uint32_t*>(rows);  // empty segments are never read
  st = launch_keys<128>(c, sg[0], count, rows, hit_flags, s, sg.data(), counts, nseg);
  if (st == FLECHE_OK) {
    c->batches++;
    c->lookups += (uint64_t)count;
  }
  return st;
}

fleche_status fleche_query_keys_seg_dev(fleche_ctx* c, const uint32_t* const* segs, const int64_t* counts_dev,
                                        int32_t world, int32_t me, float* rows, uint8_t* hit_flags,
                                        fleche_stream stream) {
  if (!c || !segs || !counts_dev || world < 1 || world > kMaxWorld || me < 0 || me >= world || !rows ||
      ((uintptr_t)rows & 15u))
    return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  if (!uniform_dims(c) || c->dv.part) return FLECHE_EINVAL;
  for (int i = 0; i < world; ++i)
    if (!segs[i]) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  st = order_on(c, s);
  if (st != FLECHE_OK) return st;
  st = launch_keys<128>(c, segs[0], 0, rows, hit_flags, s, segs, nullptr, world, counts_dev, me);
  if (st == FLECHE_OK) c->batches++;  // (the lookup count stays on the device: fleche_shard_stats)
  return st;
}

fleche_status fleche_restore_p2p_dev(fleche_ctx* c, int32_t world, const float* const* peer_rows,
                                     const uint8_t* const* peer_flags, const int64_t* counts_dev, int32_t me,
                                     float* out, fleche_stream stream) {
  if (!c || !out || ((uintptr_t)out & 15u) || !peer_rows || !counts_dev) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  if (!c->rd_ready || world < 1 || world > kMaxWorld || world != c->rd.world || me < 0 || me >= world)
    return FLECHE_EINVAL;
  PeerArgs pa;
  memset(&pa, 0, sizeof(pa));
  pa.p2p = 1;
  pa.me = me;
  pa.dcnt = counts_dev;
  for (int o = 0; o < world; ++o) {
    if (!peer_rows[o]) return FLECHE_EINVAL;
    pa.rows[o] = peer_rows[o];
    pa.flags[o] = peer_flags ? peer_flags[o] : nullptr;
  }
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  st = order_on(c, s);
  if (st != FLECHE_OK) return st;
  if (c->n <= 32) return launch_restore<32>(c, nullptr, nullptr, out, s, pa);
  if (c->n <= 128) return launch_restore<128>(c, nullptr, nullptr, out, s, pa);
  return launch_restore<FLECHE_MAX_TABLES>(c, nullptr, nullptr, out, s, pa);
}

fleche_status fleche_route_p2p(fleche_ctx* c, const int64_t* const* ids, const int64_t* lengths, int32_t world,
                               uint32_t owner_seed, uint32_t* const* peer_slots, int64_t* send_counts,
                               fleche_stream stream) {
  if (!c || !peer_slots || world < 1 || world > kMaxWorld) return FLECHE_EINVAL;
  PeerKeys pk{};
  pk.p2p = 1;
  for (int o = 0; o < world; ++o) {
    if (!peer_slots[o]) return FLECHE_EINVAL;
    pk.dst[o] = peer_slots[o];
  }
  c->route_peer = pk;
  uint32_t dummy_keys = 0;  // not written in this mode
  const fleche_status st = fleche_route(c, ids, lengths, world, owner_seed, &dummy_keys, send_counts, stream);
  c->route_peer = PeerKeys{};
  return st;
}

fleche_status fleche_restore(fleche_ctx* c, const float* rows, const uint8_t* hit_flags, float* out,
                             fleche_stream stream) {
  if (!c || !out || ((uintptr_t)out & 15u)) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  if (!c->rd_ready) return FLECHE_EINVAL;
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  st = order_on(c, s);
  if (st != FLECHE_OK) return st;
  PeerArgs pa;
  memset(&pa, 0, sizeof(pa));
  if (c->n <= 32) return launch_restore<32>(c, rows, hit_flags, out, s, pa);
  if (c->n <= 128) return launch_restore<128>(c, rows, hit_flags, out, s, pa);
  return launch_restore<FLECHE_MAX_TABLES>(c, rows, hit_flags, out, s, pa);
}

fleche_status fleche_restore_p2p(fleche_ctx* c, int32_t world, const float* const* peer_rows,
                                 const uint8_t* const* peer_flags, const int64_t* peer_off, float* out,
                                 fleche_stream stream) {
  if (!c || !out || ((uintptr_t)out & 15u) || !peer_rows || !peer_off) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  if (!c->rd_ready || world < 1 || world > kMaxWorld || world != c->rd.world) return FLECHE_EINVAL;
  PeerArgs pa;
  memset(&pa, 0, sizeof(pa));
  pa.p2p = 1;
  for (int o = 0; o < world; ++o) {
    if (!peer_rows[o] || peer_off[o] < 0) return FLECHE_EINVAL;
    pa.rows[o] = peer_rows[o];
    pa.flags[o] = peer_flags ? peer_flags[o] : nullptr;
    pa.off[o] = peer_off[o];
  }
  fleche_status st = ensure_device(c);
  if (st != FLECHE_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  st = order_on(c, s);
  if (st != FLECHE_OK) return st;
  if (c->n <= 32) return launch_restore<32>(c, nullptr, nullptr, out, s, pa);
  if (c->n <= 128) return launch_restore<128>(c, nullptr, nullptr, out, s, pa);
  return launch_restore<FLECHE_MAX_TABLES>(c, nullptr, nullptr, out, s, pa);
}

fleche_status fleche_ipc_alloc(size_t bytes, void** dptr) {
  if (!dptr || !bytes) return FLECHE_EINVAL;
  if (cudaMalloc(dptr, bytes) != cudaSuccess) {
    cudaGetLastError();
    return FLECHE_ENOMEM;
  }
  return FLECHE_OK;
}

fleche_status fleche_ipc_free(void* dptr) {
  if (!dptr) return FLECHE_EINVAL;
  return cudaFree(dptr) == cudaSuccess ? FLECHE_OK : FLECHE_ECUDA;
}

fleche_status fleche_ipc_handle(const void* dptr, uint8_t handle[64]) {
  if (!dptr || !handle) return FLECHE_EINVAL;
  static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
  cudaIpcMemHandle_t h;
  if (cudaIpcGetMemHandle(&h, (void*)dptr) != cudaSuccess) {
    cudaGetLastError();
    return FLECHE_ECUDA;
  }
  memcpy(handle, &h, 64);
  return FLECHE_OK;
}

fleche_status fleche_ipc_open(const uint8_t handle[64], void** dptr) {
  if (!handle || !dptr) return FLECHE_EINVAL;
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, 64);
  if (cudaIpcOpenMemHandle(dptr, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
    cudaGetLastError();
    return FLECHE_ECUDA;
  }
  return FLECHE_OK;
}

fleche_status fleche_ipc_close(void* dptr) {
  if (!dptr) return FLECHE_EINVAL;
  if (cudaIpcCloseMemHandle(dptr) != cudaSuccess) {
    cudaGetLastError();
    return FLECHE_ECUDA;
  }
  return FLECHE_OK;
}

fleche_status fleche_shard_stats(fleche_ctx* c, uint64_t* lookups, uint64_t* hits, uint64_t* invalid,
                                 uint64_t* unique_routed) {
  if (!c) return FLECHE_EINVAL;
  if (c->poisoned) return FLECHE_ESTATE;
  unsigned long long v[4] = {0, 0, 0, 0};
  if (c->rd_ready) {
    fleche_status st = ensure_device(c);
    if (st != FLECHE_OK) return st;
    if (c->have_last) FL_CUDA(c, cudaStreamSynchronize(c->last_stream));
    FL_CUDA(c, cudaMemcpy(v, c->rd.stats, sizeof(v), cudaMemcpyDeviceToHost));
  }
  if (lookups) *lookups = v[0];
  if (hits) *hits = v[1];
  if (invalid) *invalid = v[2];
  if (unique_routed) *unique_routed = v[3];
  return FLECHE_OK;
}

}  // extern "C"

#ifdef FLECHE_EXPERIMENTS
// timing experiments only: per-KM-warp globaltimer stamps of the last query
extern "C" __attribute__((visibility("default"))) fleche_status fleche_exp_timeline(fleche_ctx* c, uint64_t* host,
                                                                                    size_t n) {
  if (!c || !host) return FLECHE_EINVAL;
  if (c->have_last) cudaStreamSynchronize(c->last_stream);
  const size_t m = std::min(n, (size_t)c->km_blocks * 16 + 8 + 512);
  return cudaMemcpy(host, c->dv.exp_buf, m * 8, cudaMemcpyDeviceToHost) == cudaSuccess ? FLECHE_OK : FLECHE_ECUDA;
}
// host-assist threads: CLOCK_REALTIME (ns) when each thread saw the doorbell of epoch e
// and when it finished its blocks, out[(e % 64) * 2 * 64 + {0,1} * 64 + thread]
extern "C" __attribute__((visibility("default"))) fleche_status fleche_exp_ha_times(fleche_ctx* c, uint64_t* host,
                                                                                    size_t n) {
  if (!c || !host || !c->ha) return FLECHE_EINVAL;
  if (c->have_last) cudaStreamSynchronize(c->last_stream);
  memcpy(host, c->ha->exp_t, std::min(n, (size_t)64 * 2 * 64) * 8);
  return FLECHE_OK;
}
// per staging block: [KM wait start, KM flag seen, KM rows landed, KM done, early-fetch mirror,
// early-fetch copy done (GPU globaltimer), CPU published (REALTIME)]
extern "C" __attribute__((visibility("default"))) fleche_status fleche_exp_ha_blocks(fleche_ctx* c, uint64_t* host,
                                                                                     size_t nblk) {
  if (!c || !host || !c->ha) return FLECHE_EINVAL;
  if (c->have_last) cudaStreamSynchronize(c->last_stream);
  const size_t m = std::min(nblk, (size_t)c->ha->blk_cap);
  std::vector<uint64_t> g(m * 8);
  if (cudaMemcpy(g.data(), c->dv.exp_blk, m * 8 * 8, cudaMemcpyDeviceToHost) != cudaSuccess) return FLECHE_ECUDA;
  for (size_t k = 0; k < m; ++k) {
    for (int j = 0; j < 6; ++j) host[k * 7 + j] = g[k * 8 + j];
    host[k * 7 + 6] = c->ha->exp_pub[k];
  }
  return FLECHE_OK;
}
#endif
