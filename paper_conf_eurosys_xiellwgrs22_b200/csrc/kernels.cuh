// kernels.cuh — device side of the B200 flat embedding cache (sm_100a).
//
// Two kernels per one-hot batch (the paper's "1 -> 2" after decoupling):
//
//   KQ  fused, self-identified query kernel: one lane per
//       lookup; each warp finds its table from the prefix offsets in shared memory,
//       re-encodes (table, id) to a flat key, probes its 32-way set with
//       a warp-cooperative ballot (index of P:L513-528), refreshes the hit way's
//       timestamp (approximate LRU), claims each unique missed key in an
//       epoch-tagged scratch table (dedup) and appends it to its row
//       width's miss list, chains duplicate misses to their key, and copies hit rows
//       from the HBM slab into `out` with 16-byte vectors.  KQ never touches the host.
//   KM  miss kernel (unified index + replacement, P:L855-860, P:L653-666,
//       P:L985-988): each warp takes up to M unique misses of one row width, issues
//       all their zero-copy host-row loads at once (pinned, mapped host tables) and,
//       while those are in flight, admits and places each miss: victim =
//       argmin (ts, key) over ways not touched in this batch (epoch protection,
//       P:L663-666).  Rows then go to the owner's `out` position, every duplicate
//       position (restore) and the slab.  The last CTA advances the
//       device-resident epoch, so a captured CUDA graph replays correctly.
//   KP  pooling kernel (pooled queries only): bag sums of the staged
//       one-hot rows, accumulated in fp32 in bag order.
//
// Two index layouts (flat cache, Fig 5c: one pool, slabs per row width):
//   uniform (all tables share one row width d): way w of set s holds slab row 32s+w;
//           CAS on the victim's timestamp claims it, no locks.
//   bytes   (mixed widths): every set owns a set_units x 32 B region of the slab and
//           at most 32 rows whose sizes sum to <= the region; an insert evicts until
//           both limits admit the row, places it first-fit (compacting the region when
//           fragmented) under a per-set lock.  One byte budget is shared by all widths,
//           so the per-width capacity follows the workload (the flat cache's elastic
//           rescaling) with no per-class partition to tune.
#pragma once
#include <cstdint>

#ifndef FL_GATHER_F4
#define FL_GATHER_F4 8  // float4 loads per lane in flight in a row gather (A/B builds vary it)
#endif
#ifndef FL_KQ_PROBE
#define FL_KQ_PROBE 16  // index lines per lane in flight in KQ's probe (a divisor of 32): 16 = no spill with 64 registers; cfg2 KQ 36.9 vs 39.2 us at 32 (same box)
#endif
#ifndef FL_KQ_TS_DEFER
#define FL_KQ_TS_DEFER 1  // KQ consumes its timestamp-exchange result late (0 = right after it; A/B builds)
#endif
#ifndef FL_KQ_THREADS
#define FL_KQ_THREADS 128  // KQ CTA size (A/B builds: 64 with FL_KQ_MIN_BLOCKS 16 = the same warps per SM, finer CTAs)
#endif
#ifndef FL_KQ_MIN_BLOCKS
#define FL_KQ_MIN_BLOCKS 8  // KQ CTAs per SM the register budget must allow: 8 (64 regs, no spill) measured
                            // KQ 33.4 vs 35.5 us at 5 CTAs (profiles/bench_r01_kq_occupancy_*.json)
#endif

namespace fl {

constexpr uint32_t kEmpty = 0xFFFFFFFFu;
constexpr unsigned kFull = 0xFFFFFFFFu;
constexpr int kStripes = 64;  // stats counters are striped to spread L2 atomics
constexpr int kMaxCls = 6;    // row widths 8, 16, 32, 64, 128, 256 floats
constexpr int kDupSlot = 7;   // Ctl::counts column of duplicate misses
constexpr uint32_t kSlotMiss = 0xFFFFFFFFu, kSlotZero = 0xFFFFFFFEu;  // KQ -> KG codes
constexpr int kKmWarps = 4;     // KM CTA = 4 warps
constexpr int kKmStageF4 = 256; // bytes layout, per warp: staged rows of a chunk (<= 4 KB) ...
constexpr int kKmSmemF4 = 512;  // ... + the compaction buffer of one set region (<= 4 KB)
#ifndef FL_HA_BLOCK
#define FL_HA_BLOCK 64
#endif
constexpr int kHaBlock = FL_HA_BLOCK;  // host-assisted miss fetch: rows per staging block
constexpr int kHaMaxThreads = 16;  // host-assisted: at most this many host threads
constexpr int kHaSmemF4 = 512;  // host-assisted KM, per warp: 8 KB of rows landed from the host (4 KM CTAs per SM)

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
  C_HAROWS,     // host-assisted: unique misses read from the staging buffer
  C_HATIMEOUT,  // host-assisted: staging blocks not ready in time (fetched zero-copy instead)
  C_SCANS,      // watermark eviction: batches whose full-table scan ran
  kNumCtr = 16
};

struct TableInfo {
  const float* host;  // device-visible address of E_t (mapped pinned host memory)
  int64_t card;       // c_t
  uint32_t base;      // first flat key of table t (size-aware coding)
  int32_t dim;        // d_t
  int32_t cls;        // width class (index into the per-call class regions)
  uint32_t set_off;   // static per-table mode: first set of table t's partition
  uint32_t sets;      //   number of sets of the partition
  uint32_t rows;      //   capacity rows of the partition (last set may be partial)
  int64_t slab_off;   //   float offset of the partition's rows in the slab
  uint32_t hmask;     // short flat keys (R24): 2^g_t - 1 for a hashed table
  int32_t hashed;     //   1 = feature IDs of this table are hashed into g_t bits
};

// Short flat keys ("feature ID (hashed) bits", reading R24): the
// hashed feature ID of table t, splitmix64(id ^ (t << 48) ^ 0x6A09E667F3BCC909) mod 2^g.
__device__ __forceinline__ int64_t short_feature_id(int t, int64_t id, uint32_t hmask) {
  uint64_t z = ((uint64_t)id ^ ((uint64_t)t << 48) ^ 0x6A09E667F3BCC909ull) + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return (int64_t)((z ^ (z >> 31)) & (uint64_t)hmask);
}

struct MissRec {  // one unique missed key (its owner lookup)
  int64_t off;    // float offset of the owner's row in `out`
  uint32_t fk;    // flat key
  uint32_t scr;   // scratch slot of the key (head of its duplicate chain)
  int32_t t;      // table
  int32_t pad;
  uint64_t hst;   // host-assisted: float offset of the row's staging slot (kNoStage: read the table)
};
constexpr unsigned long long kNoStage = ~0ull;

struct DupRec {  // a later occurrence of a missed key in the same batch
  int64_t off;   // float offset of the duplicate's row in `out`
  uint32_t scr;  // scratch slot of the key -> its owner's row (owner_off)
  int32_t dim;   // row width
};

struct Ctl {
  uint32_t epoch;  // current batch epoch (1-based); advanced by the last KM CTA
  uint32_t done;   // KM grid barrier arrivals (before the restore)
  uint32_t done2;  // KM CTA arrivals at the end (the last one closes the batch)
  uint32_t err_invalid;
  uint32_t ha_rung;  // host-assisted: epoch whose doorbell KQ's last CTA has rung
  uint32_t counts[2][8];  // [epoch & 1][class 0..5: unique misses; 7: duplicate misses]
  long long occ_bytes;    // row bytes currently cached
  uint32_t ke_done;       // watermark eviction: KE2 CTA arrival counter
  uint32_t km_bar;        // KM grid barrier: epoch whose owner rows are all in `out`
  long long ke_occ;
  uint32_t kq_done;       // host-assisted: KQ CTA arrivals (the last one rings the doorbell)
  uint32_t kq_end;        // early fetch: epoch whose KQ lookup CTAs have all finished (counts final)
  uint32_t kq_end_pad;
  uint32_t ha_abort;      // host-assisted: epoch whose staging the poller gave up on (timeout)
  // unified-index share tuning (see ui_tune): the host threads' share of a
  // batch's staging blocks (x 2^-16; the GPU's zero-copy reads -- the unified index -- take
  // the rest), and the loop's state
  uint32_t ha_frac_q16;
  uint32_t tune_phase;         // 0 = growing the unified-index share, 1 = paused at the peak
  unsigned long long km_t0;    // globaltimer at this batch's KM start (CTA 0)
  unsigned long long win_ns;   // current window: KM time summed
  unsigned long long win_miss; //   unique misses summed
  uint32_t win_n;              //   batches
  uint32_t tune_since;         // paused: windows since the last probe
  double prev_cost;            // ns per unique miss of the previous window (growing) / at the peak (paused)
  uint32_t tune_best;          // probing: the share to return to
  int32_t tune_dir;            // probing: direction of the next probe (+1 / -1 share step)       // watermark eviction: occ_bytes as KE1 saw it (KE2's one snapshot per scan)
};

// Host-assisted miss fetch (FLECHE_FLAG_HOST_ASSIST): the CPU-DRAM layer's threads
// gather missed rows (Fig 8b) -- host cores read scattered rows without the
// GPU's address-translation limit on scattered zero-copy reads (profiles/), and the GPU
// then reads their staging buffer contiguously.  The owner lane of each unique miss in KQ
// writes (table, row, staging slot) to the request list in pinned host memory at its
// miss-list index; KQ's last warp rings a doorbell with the batch's per-width miss counts.
// Host thread i gathers every staging block k (kHaBlock list indices) with k % T == i, in
// increasing k, and sets each block's ready word (= epoch) once staged.  ONE poller warp of KM reads the batch's
// ready words over the link (32 per load instruction) and mirrors them into HBM; every
// other KM warp waits on the mirror for its block (no per-block polls competing with the
// row reads for the link), then reads the block's staged rows.  When no new block has
// been staged for kHaStallNs (a host thread descheduled mid-batch) or past the timeout,
// the poller gives up and the waiting readers fetch their rows zero-copy from the tables,
// so a missing or slow host thread costs time, never correctness.  Every area is double-buffered by
// epoch parity.
struct HaReq {  // one request, both halves tagged with the batch epoch (see ha_req_make)
  unsigned long long tid;    // table (9 bits) << 55 | epoch (15 bits) << 40 | row (40 bits)
  unsigned long long stage;  // epoch (24 bits) << 40 | float offset of its staging slot (40 bits; all ones: none)
};
constexpr unsigned long long kReqLow40 = (1ull << 40) - 1;
// KQ writes a request with one 16-byte store and no system fence: the host thread that
// reads it after the doorbell re-reads until both halves carry the batch's epoch tags, so a
// request still in flight over the link (or a torn read) is never taken for this batch's.
__host__ __device__ __forceinline__ HaReq ha_req_make(int t, int64_t id, uint64_t stage, uint32_t epoch) {
  return HaReq{((unsigned long long)t << 55) | ((unsigned long long)(epoch & 0x7FFFu) << 40) | ((uint64_t)id & kReqLow40),
               ((unsigned long long)(epoch & 0xFFFFFFu) << 40) | (stage & kReqLow40)};
}
__host__ __device__ __forceinline__ bool ha_req_current(const HaReq& r, uint32_t epoch) {
  return (uint32_t)((r.tid >> 40) & 0x7FFFu) == (epoch & 0x7FFFu) && (uint32_t)(r.stage >> 40) == (epoch & 0xFFFFFFu);
}
struct HaDesc {            // written by the doorbell ringer, read by the host threads
  uint32_t epoch;
  uint32_t cnt[8];         // unique misses of width class c this batch
  uint32_t hcut[8];        // split: the host threads stage class c's blocks < hcut[c], KM reads the rest itself
  uint32_t pad;
  uint32_t epoch2;         // = epoch, written last: the host accepts the descriptor once both match
};

struct Dev {
  uint32_t* keys;   // [sets][32] flat keys, kEmpty = free way
  uint32_t* ts;     // [sets][32] batch epoch of last touch (0 = never)
  uint16_t* loc;    // bytes layout: [sets][32] (size units << 8 | offset units), 32 B units
  uint32_t* lock;   // bytes layout: [sets] insert locks
  float* slab;      // uniform: [sets*32][dim];  bytes: [sets][set_units * 8]
  unsigned long long* scratch;   // [scr_mask+1] (epoch << 32 | fk) dedup tags
  int64_t* owner_off;            // [scr_mask+1] float offset in `out` of the key's owner row
  unsigned long long* firstpos;  // [scr_mask+1] (~epoch << 32 | first occurrence of the key in the batch)
  unsigned long long* ipos;      // uniform layout: [sets][32] (epoch << 32 | inserter's first occurrence << 1 | busy)
  MissRec* miss;                 // [max_lookups], split into per-class regions per call
  DupRec* dup;                   // [max_lookups]
  Ctl* ctl;
  unsigned long long* stats;  // [kStripes][kNumCtr]
  const TableInfo* tables;    // [n]
  uint32_t sets, rows, scr_mask, hash_seed;
  int32_t dim, admit_all;     // dim: row width of the uniform layout (bytes layout: the widest row)
  uint64_t admit_thr, admit_seed;
  int32_t bytes;     // 0 = uniform layout, 1 = bytes layout
  uint32_t set_units;  // bytes layout: region of a set in 32 B units (<= 256)
  int32_t part;      // static per-table partitions (HugeCTR-like baseline, NEXT-1)
  int32_t ntables;
  const uint64_t* kdec;  // [ntables] (base_t << 16 | t) sorted by base: flat key -> table
  // address-ordered miss scratch (uniform layout): a missed key's first scratch slot is
  // monotone in its host-row address, slot0 = ((addr - host_lo) * host_mul) >> 64, so KM
  // can hand each warp a contiguous address window (host-link reads in address order)
  int32_t ordered;
  int32_t bands;     // ordered: band-major sweep, ~bands misses per warp per band (0: M; < 0: off)
  uint64_t host_lo, host_mul;
  // host-assisted miss fetch (mapped pinned host memory; see HaReq)
  int32_t ha;                  // 1 = host-assisted miss fetch on
  int32_t ha_pad;
  HaReq* ha_req;               // [2][ha_req_cap]: indexed like the miss list
  HaDesc* ha_desc;             // [2]
  unsigned long long* ha_bell; // doorbell: epoch of the latest published descriptor
  unsigned long long* ha_start;  // start word: epoch of the batch whose KQ has begun (host threads stream its requests)
  uint32_t* ha_ready;          // [2][ha_blk_cap] (host memory) epoch of each staging block once staged
  uint32_t* ha_seen;           // [ha_blk_cap] (HBM) the poller warp's mirror of ha_ready[epoch & 1]
  float* ha_stage;             // [2][ha_stage_floats]
  float* ha_hstage;            // early fetch: [2][ha_stage_floats] (HBM) copy of the staged blocks
  HaReq* ha_reqd;              // request forwarding: [ha_req_cap] (HBM) KQ's requests before they go to the host
  uint32_t* ha_hseen;          // early fetch: [ha_blk_cap] (HBM) epoch once a block's rows are in ha_hstage
  uint32_t ha_req_cap, ha_blk_cap;  // staging rows (= request slots) and blocks per epoch parity
  uint32_t ha_rbase[8];        // first staging row of width class c (a multiple of kHaBlock)
  uint32_t ha_rcap[8];         // staging rows of class c (a multiple of kHaBlock): its misses beyond go zero-copy
  uint32_t ha_row_floats;      // stride of a staging row (the widest row)
  uint32_t ha_pad3;
  uint64_t ha_stage_floats;
  uint64_t ha_timeout_ns;
  uint32_t ha_frac_fixed;      // 1 = FLECHE_HA_FRAC fixed the host threads' share (no tuning loop)
  uint32_t ha_min_rows;        // batches with fewer unique misses stay all zero-copy (the split loses there)
  uint32_t ha_unit_pieces;     // KM work unit = this many 16-row pieces (0: adaptive to the batch)
  uint32_t ha_kf_tail;         // early fetch: 1 = the fetch CTAs copy every host block (KQ ends after them), 0 = stop with the lookups
#ifdef FLECHE_EXPERIMENTS
  int32_t exp_mode;  // timing experiments only (libfleche_exp.so); breaks semantics
  int32_t exp_pad;
  unsigned long long* exp_buf;  // per KM warp: globaltimer at start / rows landed / end
  uint32_t exp_slots;           // exp_buf[exp_slots]: KQ's doorbell time (host-assisted)
  uint32_t exp_pad2;
  unsigned long long* exp_blk;  // host-assisted KM, per staging block: wait start / flag seen / rows landed / done
#endif
};

template <int MAXT>
struct QArgs {
  const int64_t* ids[MAXT];  // per-table device ID arrays
  int64_t scan[MAXT + 1];    // exclusive prefix of lengths
  int64_t out_off[MAXT];     // float offset of O_t in out
  int64_t cls_off[8];        // start of each class's region of the miss list
  float* out;
  int64_t g0;                // batch position of this launch's first lookup (per-table launches)
  const uint32_t* fkeys;     // key-sharded owner side: flat keys instead of per-table IDs
  uint8_t* hit_flags;        // optional per-lookup hit flags (key-sharded)
  uint32_t* slots;           // decoupled copy: per-lookup hit slot / kSlotMiss / kSlotZero for KG
  int32_t n;
  int32_t t0;                // first table of this launch (per-table launches: t0 = t, n = 1)
  int32_t fkseg;             // key-sharded fused exchange: fkeys come in n segments (ids[], scan[])
  int32_t ha_bell;           // host-assisted: the last CTA rings the host threads' doorbell
  int32_t ncls;              //   (number of width classes of the miss list)
  const int64_t* dcnt;       // key-sharded sync-free: [n][n] routed-count matrix in device memory
  int32_t dme;               //   this rank (segment i's count = dcnt[i * n + dme])
  int32_t nfetch;            // early fetch: CTAs 0..nfetch-1 copy staged blocks into HBM (kq_fetch)
  int32_t nfwd;              // request forwarding: the next nfwd CTAs move requests to the host (kq_forward)
  int32_t pad4;
  int32_t cls_dim[8];        //   (row width of each class)
};

struct KMArgs {
  float* out;
  int64_t cls_off[8];
  int32_t cls_dim[8];
  int32_t ncls;
  int32_t bell;  // host-assisted: KM (not KQ's last CTA) rings the doorbell
};

template <int MAXT>
struct PArgs {                  // pooling: column slots of table t = bags_t * d_t / 4
  const int64_t* offs[MAXT];    // CSR bag offsets of table t (device), bags_t + 1 entries
  int64_t cscan[MAXT + 1];      // exclusive prefix of column slots
  int64_t stage_off[MAXT];      // float offset of table t's staged rows
  int64_t out_off[MAXT];        // float offset of table t's pooled rows in out
  const float* stage;
  float* out;
  int32_t n;
  int32_t pad;
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
// Static per-table mode: table t's keys live only in its own partition of sets.
__device__ __forceinline__ uint32_t set_of_t(const Dev& dv, const TableInfo* ti, uint32_t fk) {
  return dv.part ? ti->set_off + __umulhi(fmix32(fk ^ dv.hash_seed), ti->sets) : set_of(dv, fk);
}
__device__ __forceinline__ int ways_in_t(const Dev& dv, const TableInfo* ti, uint32_t s) {
  if (!dv.part) return ways_in(dv, s);
  const uint32_t lo = (s - ti->set_off) * 32u;
  return ti->rows <= lo ? 0 : (ti->rows - lo >= 32u ? 32 : (int)(ti->rows - lo));
}
// Uniform layout: slab row of a slot (global slot = 32 * set + way).
__device__ __forceinline__ float* slot_row(const Dev& dv, const TableInfo* ti, uint32_t slot, int d) {
  return dv.part ? dv.slab + ti->slab_off + (size_t)(slot - ti->set_off * 32u) * (size_t)d
                 : dv.slab + (size_t)slot * (size_t)d;
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
__device__ __forceinline__ float4 ld_cg_v4(const float* p) {
  float4 v;
  asm volatile("ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p) : "memory");
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
__device__ __forceinline__ uint32_t ld_cg_u16(const uint16_t* p) {
  unsigned short v;
  asm volatile("ld.global.cg.u16 %0, [%1];" : "=h"(v) : "l"(p) : "memory");
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
// System-scope accesses to the host-assisted areas (written by host threads while the
// kernel runs: strong loads, never a stale L1/L2 copy; the ready flag is an acquire).
__device__ __forceinline__ uint32_t ld_acquire_sys_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
// Staging rows: weak loads that coalesce into full-line link reads, but never hit a
// stale L2 copy of system memory (.cv: discard a matching L2 line, fetch again); their
// freshness w.r.t. the host's writes comes from the block's acquire of the ready flag.
__device__ __forceinline__ float4 ld_cv_v4(const float* p) {
  float4 v;
  asm volatile("ld.global.cv.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Poll of a host-written flag: .cv discards a matching (possibly stale) L2 copy of the
// system-memory line and fetches it again over the link.
__device__ __forceinline__ uint32_t ld_cv_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.global.cv.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
// Grid barrier helpers (KM is a cooperative launch: every CTA is resident at once).
__device__ __forceinline__ uint32_t ld_acquire_gpu_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ unsigned long long ld_acquire_sys_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_cv_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.global.cv.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_acquire_gpu_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Host-assisted geometry.  Staging row r = ha_rbase[c] + j holds the j-th unique miss of
// width class c (its class-local miss-list index), for j < ha_rcap[c]; block b = r / 64 is
// always the same 64 rows of staging memory, owned by host thread b % T in every batch
// (a stalled thread can only ever rewrite its own blocks, whatever the batch geometry).
// The host threads take class c's blocks below hcut (its share of the class's staged rows).
__host__ __device__ __forceinline__ uint32_t ha_hcut(uint32_t cnt, uint32_t rcap, uint32_t frac_q16) {
  const uint32_t nb = ((cnt < rcap ? cnt : rcap) + kHaBlock - 1) / kHaBlock;
  return (uint32_t)(((unsigned long long)nb * frac_q16 + 65535ull) >> 16);
}

// The poller warp: mirror the ready words of staging blocks [kb0, kend) into HBM until all
// are staged, or give up (ha_abort = epoch: the readers still waiting go zero-copy) when
// no new block became ready for kHaStallNs after one did (a host thread descheduled
// mid-batch), or past the timeout.  Each round reads the ready words of every block not
// mirrored yet (strong relaxed loads, 4 per lane in flight), then one system-scope fence
// orders the staged rows of the newly ready blocks before their mirror words.
constexpr unsigned long long kHaStallNs = 150000;
__device__ __forceinline__ uint32_t ld_relaxed_sys_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
// Ready words of the batch's host blocks: class c's blocks [rbase_c / 64, + hcut_c).
struct HaBlocks {
  uint32_t lo[8], n[8];
  int ncls;
};
__device__ __forceinline__ void ha_poll(const Dev& dv, uint32_t epoch, const HaBlocks& hb, int lane) {
  const uint32_t* ready = dv.ha_ready + (size_t)(epoch & 1u) * dv.ha_blk_cap;
  const unsigned long long t0 = globaltimer_ns();
  unsigned long long t_progress = 0;  // last time a new block was seen ready (0: none yet)
  uint32_t lo[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) lo[c] = c < hb.ncls ? hb.lo[c] : 0u;  // class c: blocks below lo[c] mirrored
  while (true) {
    if (*(volatile uint32_t*)&dv.ctl->ha_abort == epoch) break;  // given up already (early fetch's poller)
    uint32_t fresh = 0, missing = 0;
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      if (c >= hb.ncls) continue;
      const uint32_t kend = hb.lo[c] + hb.n[c];
      uint32_t first_missing = kend;
      for (uint32_t k0 = lo[c]; k0 < kend; k0 += 32 * 4) {
        uint32_t v[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const uint32_t k = k0 + 32 * q + lane;
          v[q] = (k < kend && ld_acquire_gpu_u32(dv.ha_seen + k) != epoch) ? ld_relaxed_sys_u32(ready + k) : ~0u;
        }
        uint32_t newly = 0;
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const uint32_t k = k0 + 32 * q + lane;
          if (v[q] == epoch) newly |= 1u << q;
          const unsigned miss = __ballot_sync(kFull, k < kend && v[q] != ~0u && v[q] != epoch);
          if (miss) first_missing = min(first_missing, k0 + 32 * q + (uint32_t)(__ffs(miss) - 1));
        }
        if (__any_sync(kFull, newly)) {
          asm volatile("fence.acq_rel.sys;" ::: "memory");  // the rows staged before these ready words
#pragma unroll
          for (int q = 0; q < 4; ++q)
            if (newly & (1u << q)) st_release_gpu_u32(dv.ha_seen + k0 + 32 * q + lane, epoch);
          fresh += __popc(__ballot_sync(kFull, newly != 0));
        }
      }
      lo[c] = first_missing;
      if (first_missing < kend) missing = 1;
    }
    if (!missing) break;
    const unsigned long long now = globaltimer_ns();
    if (fresh) t_progress = now;
    if (now - t0 > dv.ha_timeout_ns || (t_progress && now - t_progress > kHaStallNs)) {
      if (lane == 0) st_release_gpu_u32(&dv.ctl->ha_abort, epoch);
      break;
    }
  }
}

// A reader warp's wait (one lane) for staging block kb; false: timed out / abandoned.
__device__ __forceinline__ bool ha_wait_block(const Dev& dv, uint32_t epoch, uint32_t kb) {
  const unsigned long long t0 = globaltimer_ns();
  while (true) {
    if (ld_acquire_gpu_u32(dv.ha_seen + kb) == epoch) return true;
    if (*(volatile uint32_t*)&dv.ctl->ha_abort == epoch) return false;
    if (globaltimer_ns() - t0 > dv.ha_timeout_ns + 20000ull) return false;  // safety net behind the poller's
    __nanosleep(64);
  }
}

// Host-assisted split: the host threads gather the first ceil(frac * nblocks) staging
// blocks of every class while KM's other warps read the rest zero-copy from the tables at
// the same time (two independent paths to the rows: host cores + contiguous link reads,
// and the GPU's own translated reads).
// Host-assisted fetch active for this batch: enough unique misses (FLECHE_HA_MIN_ROWS) and
// a non-zero share.  Otherwise KM takes the plain (address-ordered) zero-copy path and the
// host threads are not woken.
__device__ __forceinline__ bool ha_active(const Dev& dv, const KMArgs& ka, int par) {
  if (!dv.ha || !*(volatile uint32_t*)&dv.ctl->ha_frac_q16) return false;
  uint32_t total = 0;
  for (int c = 0; c < ka.ncls; ++c) total += *(volatile uint32_t*)&dv.ctl->counts[par][c];
  return total >= dv.ha_min_rows;
}

// Programmatic dependent launch (sm_90+): the batch's kernels are launched with
// programmatic stream serialization, so a kernel's launch and prologue overlap the tail
// of its predecessor; pdl_wait() (griddepcontrol.wait) then blocks until the
// predecessor grid has completed and its writes are visible.  No-ops otherwise.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ unsigned long long warp_min_u64(unsigned long long x) {
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    const unsigned long long y = __shfl_xor_sync(kFull, x, o);
    x = y < x ? y : x;
  }
  return x;
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
  constexpr int CH0 = (FL_GATHER_F4 / VPL) > 0 ? (FL_GATHER_F4 / VPL) : 1;
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

// Same copy with rows in shared memory (generic loads): row r of the warp at src[lane r].
template <int D>
__device__ __forceinline__ void copy_rows_generic(const float* src, float* dst, int lane) {
  constexpr int VEC = D / 4;
  constexpr int LPR = VEC < 32 ? VEC : 32;
  constexpr int RPP = 32 / LPR;
  constexpr int VPL = VEC / LPR;
  constexpr int PASSES = 32 / RPP;
  const int sub = lane % LPR, rs = lane / LPR;
#pragma unroll 4
  for (int p = 0; p < PASSES; ++p) {
    const int r = p * RPP + rs;
    const float* s = (const float*)__shfl_sync(kFull, (unsigned long long)src, r);
    float* o = (float*)__shfl_sync(kFull, (unsigned long long)dst, r);
    if (o) {
#pragma unroll
      for (int k = 0; k < VPL; ++k)
        st_v4(o + 4 * (sub + k * LPR), *reinterpret_cast<const float4*>(s + 4 * (sub + k * LPR)));
    }
  }
}

// Fallback for warps whose lanes have different row widths: one row at a time.
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

// Row gather for the warp's 32 lanes, specialised when every active lane has the same width.
__device__ __forceinline__ void gather_dispatch(const float* src, float* dst, int d, bool active, int lane) {
  const int d0 = __shfl_sync(kFull, d, 0);
  const bool uni = __all_sync(kFull, !active || d == d0);
  if (uni && d0 == 32) gather_rows<32>(src, dst, lane);
  else if (uni && d0 == 64) gather_rows<64>(src, dst, lane);
  else if (uni && d0 == 128) gather_rows<128>(src, dst, lane);
  else if (uni && d0 == 16) gather_rows<16>(src, dst, lane);
  else if (uni && d0 == 8) gather_rows<8>(src, dst, lane);
  else if (uni && d0 == 256) gather_rows<256>(src, dst, lane);
  else gather_rows_any(src, dst, d, lane);
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
  // row r -> smem[r * VEC ...]
  __device__ __forceinline__ void to_smem(float4* sm, int lane) const {
    const int sub = lane % LPR, rs = lane / LPR;
#pragma unroll
    for (int p = 0; p < PASSES; ++p) {
      const int r = p * RPP + rs;
      if (r < M) {
#pragma unroll
        for (int k = 0; k < VPL; ++k) sm[r * VEC + sub + k * LPR] = v[p][k];
      }
    }
  }
};

// Bulk-copy (TMA engine) helpers for KQ's hit gather (TD > 0): rows land in shared memory
// through cp.async.bulk with an mbarrier transaction count; the warp's contiguous output
// block leaves with one bulk store.
__device__ __forceinline__ void mbar_init(unsigned mb, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(mb), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned mb, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned mb, unsigned parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tKQ_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra KQ_WAIT_%=;\n\t}" ::"r"(mb), "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* smem, const void* gmem, unsigned bytes, unsigned mb) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   (unsigned)__cvta_generic_to_shared(smem)),
               "l"(gmem), "r"(bytes), "r"(mb)
               : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* gmem, const void* smem, unsigned bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gmem),
               "r"((unsigned)__cvta_generic_to_shared(smem)), "r"(bytes)
               : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}

// Request forwarding (host-assisted): KQ's owner lanes write their 16-byte requests into HBM
// and qa.nfwd CTAs of KQ move them to the host threads' pinned request list a staging block
// (64 requests, 1 KiB) at a time, coalesced.  The lookups themselves then never store to
// system memory: scattered 16-byte posted writes over the link cost KQ +6 us at cfg2 and
// +100 us at cfg4, and on some boxes of the pool they stalled whole KQ launches for 0.2-0.4
// ms (ncu launch list, profiles/r02b).  A forwarder warp takes class-local blocks w, w + W,
// ...: a block goes once all its requests carry this batch's tags (the last partial block
// once the last lookup CTA has published the counts, ctl->kq_end); the host threads wait on
// the same tags, so nothing else changes for them.  Bounded: after the counts are known, a
// block that makes no progress for kFwdStallNs is left to the host threads' own timeout.
constexpr unsigned long long kFwdStallNs = 200000;
template <int MAXT>
__device__ __forceinline__ void kq_forward(const QArgs<MAXT>& qa, const Dev& dv) {
  const int lane = threadIdx.x & 31;
  const uint32_t W = (uint32_t)qa.nfwd * (blockDim.x >> 5);
  const uint32_t w = (blockIdx.x - (uint32_t)qa.nfetch) * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const uint32_t epoch = *(volatile uint32_t*)&dv.ctl->epoch;
  const int par = epoch & 1u;
  HaReq* hreq = dv.ha_req + (size_t)par * dv.ha_req_cap;
  uint32_t cur[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) cur[c] = w;
  unsigned long long t_prog = 0;
  while (true) {
    const bool known = ld_acquire_gpu_u32(&dv.ctl->kq_end) == epoch;
    if (known && *(volatile uint32_t*)&dv.ctl->ha_rung != epoch) return;  // not a host-assisted batch
    bool left = false, prog = false;
#pragma unroll 1
    for (int c = 0; c < qa.ncls; ++c) {
      const uint32_t rcap = dv.ha_rcap[c];
      const uint32_t nrow = known ? min(*(volatile uint32_t*)&dv.ctl->counts[par][c], rcap) : rcap;
      const uint32_t nb = known ? (nrow + kHaBlock - 1) / kHaBlock : rcap / kHaBlock;
      if (cur[c] >= nb) continue;
      left = true;
      const uint32_t lim = known ? min((uint32_t)kHaBlock, nrow - cur[c] * kHaBlock) : (uint32_t)kHaBlock;
      const size_t r0 = (size_t)dv.ha_rbase[c] + (size_t)cur[c] * kHaBlock;
      bool ok = true;
      HaReq q[kHaBlock / 32 > 0 ? kHaBlock / 32 : 1];
#pragma unroll
      for (int h = 0; h < (kHaBlock + 31) / 32; ++h) {
        const uint32_t i = h * 32 + lane;
        if (i < lim) {
          asm volatile("ld.global.cg.v2.u64 {%0, %1}, [%2];" : "=l"(q[h].tid), "=l"(q[h].stage) : "l"(dv.ha_reqd + r0 + i));
          ok = ok && ha_req_current(q[h], epoch);
        }
      }
      if (__all_sync(kFull, ok)) {
#pragma unroll
        for (int h = 0; h < (kHaBlock + 31) / 32; ++h) {
          const uint32_t i = h * 32 + lane;
          if (i < lim)
            asm volatile("st.global.v2.u64 [%0], {%1, %2};" ::"l"(hreq + r0 + i), "l"(q[h].tid), "l"(q[h].stage) : "memory");
        }
        cur[c] += W;
        prog = true;
      }
    }
    if (!left) return;
    if (known) {
      const unsigned long long now = globaltimer_ns();
      if (prog || !t_prog) t_prog = now;
      else if (now - t_prog > kFwdStallNs) return;
    }
    if (!prog) __nanosleep(100);
  }
}

// Early fetch (host-assisted): the first qa.nfetch CTAs of KQ do no lookups; they move the
// batch's staged blocks over the link into HBM WHILE the other CTAs are still indexing, so
// the link is busy during KQ instead of only during KM (the host threads stream the
// requests as KQ writes them).  Warp 0 of CTA 0 mirrors the host threads' ready words into
// ha_seen (as KM's poller does); every other warp copies its static share of each width
// class's blocks (class-local block b = w, w + W, ...) as they become ready, and publishes
// ha_hseen[kb] = epoch; KM then reads those rows from HBM.  The batch's block counts are
// known once the last lookup CTA has rung the doorbell (ctl->kq_end = epoch); the fetch
// CTAs stop at the host share (hcut) or give up (ha_abort) when the host threads stall, and
// KM fetches whatever is not in HBM exactly as without early fetch.
constexpr unsigned long long kKfStallNs = 150000;
template <int MAXT>
__device__ __forceinline__ void kq_fetch(const QArgs<MAXT>& qa, const Dev& dv) {
  const int lane = threadIdx.x & 31;
  const uint32_t w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const uint32_t nwk = (uint32_t)qa.nfetch * (blockDim.x >> 5) - 1u;  // copy warps
  const uint32_t epoch = *(volatile uint32_t*)&dv.ctl->epoch;
  const int par = epoch & 1u;
  const int ncls = qa.ncls;
  const uint32_t* ready = dv.ha_ready + (size_t)par * dv.ha_blk_cap;
  const float* stage = dv.ha_stage + (size_t)par * dv.ha_stage_floats;
  float* hstage = dv.ha_hstage + (size_t)par * dv.ha_stage_floats;
  // the batch's host share per class, once every lookup CTA has finished (0xFFFFFFFF before)
  auto share = [&](int c, bool& known, bool& active) -> uint32_t {
    if (ld_acquire_gpu_u32(&dv.ctl->kq_end) != epoch) {
      known = false;
      return 0xFFFFFFFFu;
    }
    known = true;
    active = *(volatile uint32_t*)&dv.ctl->ha_rung == epoch;
    if (!active || !dv.ha_kf_tail) return 0u;  // default: stop with the lookups (KM takes the rest)
    const uint32_t cnt = *(volatile uint32_t*)&dv.ctl->counts[par][c];
    return ha_hcut(cnt, dv.ha_rcap[c], *(volatile uint32_t*)&dv.ctl->ha_frac_q16);
  };
  if (w == 0) {  // the poller: ready words -> ha_seen (a window of 128 blocks per class ahead)
    uint32_t lo[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) lo[c] = 0;  // class-local: blocks below lo[c] mirrored
    unsigned long long t_prog = globaltimer_ns();
    while (true) {
      if (*(volatile uint32_t*)&dv.ctl->ha_abort == epoch) return;
      bool known = false, active = true, left = false, fresh = false;
#pragma unroll 1
      for (int c = 0; c < ncls; ++c) {
        const uint32_t b0 = dv.ha_rbase[c] / kHaBlock, nb = min(share(c, known, active), dv.ha_rcap[c] / kHaBlock);
        if (lo[c] >= nb) continue;
        left = true;
        const uint32_t b = lo[c] + 4u * lane;
        uint32_t v[4];
#pragma unroll
        for (int q = 0; q < 4; ++q)
          v[q] = (b + q < nb && b + q < lo[c] + 128u && ld_acquire_gpu_u32(dv.ha_seen + b0 + b + q) != epoch)
                     ? ld_relaxed_sys_u32(ready + b0 + b + q)
                     : epoch;
        unsigned newly = 0;
#pragma unroll
        for (int q = 0; q < 4; ++q)
          if (b + q < nb && b + q < lo[c] + 128u && v[q] == epoch) newly |= 1u << q;
        if (__any_sync(kFull, newly)) {
          asm volatile("fence.acq_rel.sys;" ::: "memory");  // the rows staged before these ready words
#pragma unroll
          for (int q = 0; q < 4; ++q)
            if (newly & (1u << q)) {
              st_release_gpu_u32(dv.ha_seen + b0 + b + q, epoch);
#ifdef FLECHE_EXPERIMENTS
              if (dv.exp_blk) dv.exp_blk[(b0 + b + q) * 8 + 4] = globaltimer_ns();
#endif
            }
        }
        // advance past the mirrored prefix
        const unsigned all4 = __ballot_sync(kFull, b >= nb || b >= lo[c] + 128u ||
                                                       (v[0] == epoch && v[1] == epoch && v[2] == epoch && v[3] == epoch));
        const uint32_t adv = all4 == kFull ? 128u : 4u * (uint32_t)(__ffs(~all4) - 1);
        if (adv) fresh = true;
        lo[c] = min(nb, lo[c] + adv);
        if (lo[c] < nb) left = true;
      }
      if (!left && known) return;
      if (known && !active) return;
      const unsigned long long now = globaltimer_ns();
      if (fresh) t_prog = now;
      if (known && now - t_prog > kKfStallNs) {  // a host thread stalled: KM takes over (zero-copy)
        if (lane == 0) st_release_gpu_u32(&dv.ctl->ha_abort, epoch);
        return;
      }
      __nanosleep(200);
    }
  }
  // copy warps: class-local blocks b = w - 1 + k * nwk of every class, as they become ready
  uint32_t cur[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) cur[c] = w - 1u;
  while (true) {
    if (*(volatile uint32_t*)&dv.ctl->ha_abort == epoch) return;
    bool left = false, progressed = false;
#pragma unroll 1
    for (int c = 0; c < ncls; ++c) {
      bool known = false, active = true;
      const uint32_t nb = min(share(c, known, active), dv.ha_rcap[c] / kHaBlock);
      if (cur[c] >= nb) continue;
      left = true;
      const uint32_t kb = dv.ha_rbase[c] / kHaBlock + cur[c];
      if (ld_acquire_gpu_u32(dv.ha_seen + kb) != epoch) continue;
      // the block's rows: host staging -> HBM (row stride ha_row_floats, class width D)
      const int D = qa.cls_dim[c];
      const uint32_t vec = (uint32_t)D / 4u, n4 = (uint32_t)kHaBlock * vec;
      const size_t base = (size_t)kb * kHaBlock * dv.ha_row_floats;
      bool quit = false;
#pragma unroll 1
      for (uint32_t q0 = 0; q0 < n4; q0 += 32u * 8u) {
        if (!dv.ha_kf_tail && ld_acquire_gpu_u32(&dv.ctl->kq_end) == epoch) {  // lookups done: KM takes over
          quit = true;
          break;
        }
        float4 v[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const uint32_t q = q0 + 32u * i + lane;
          v[i] = q < n4 ? ld_cv_v4(stage + base + (size_t)(q / vec) * dv.ha_row_floats + 4u * (q % vec))
                        : make_float4(0.f, 0.f, 0.f, 0.f);
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const uint32_t q = q0 + 32u * i + lane;
          if (q < n4) st_v4(hstage + base + (size_t)(q / vec) * dv.ha_row_floats + 4u * (q % vec), v[i]);
        }
      }
      __syncwarp();
      if (quit) return;
      if (lane == 0) {
        __threadfence();
        st_release_gpu_u32(dv.ha_hseen + kb, epoch);
#ifdef FLECHE_EXPERIMENTS
        if (dv.exp_blk) dv.exp_blk[kb * 8 + 5] = globaltimer_ns();
#endif
      }
      cur[c] += nwk;
      progressed = true;
    }
    if (!left) return;
    if (!progressed) __nanosleep(200);
  }
}

// KQ's side CTAs: [0, nfetch) early fetch, [nfetch, nfetch + nfwd) request forwarding (one
// call site, so the lookup path keeps its registers)
template <int MAXT>
__device__ __forceinline__ void kq_side(const QArgs<MAXT>& qa, const Dev& dv) {
  if ((int)blockIdx.x < qa.nfetch) kq_fetch<MAXT>(qa, dv);
  else kq_forward<MAXT>(qa, dv);
}

// TD > 0: hit rows gathered with bulk copies through TD-float shared-memory rows (one row
// width for every table; dynamic shared memory = 4 warps x 32 rows x TD floats).
template <int MAXT, int TD>
__global__ void __launch_bounds__(FL_KQ_THREADS, FL_KQ_MIN_BLOCKS) kq_kernel(const __grid_constant__ QArgs<MAXT> qa,
                                                                   const __grid_constant__ Dev dv) {
  __shared__ int64_t s_scan[MAXT + 1];
  __shared__ __align__(8) unsigned long long s_mbar[4];
  extern __shared__ __align__(128) float kq_dyn[];
  if (!qa.dcnt)
    for (int i = threadIdx.x; i <= qa.n; i += blockDim.x) s_scan[i] = qa.scan[i];
  if constexpr (TD > 0) {
    if (threadIdx.x < 4) mbar_init((unsigned)__cvta_generic_to_shared(&s_mbar[threadIdx.x]), 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  pdl_wait();  // the previous batch (or the caller's producer of ids) has completed
  if ((int)blockIdx.x < qa.nfetch + qa.nfwd) {  // early-fetch / request-forwarding CTA (no lookups)
    kq_side<MAXT>(qa, dv);
#ifdef FLECHE_EXPERIMENTS
    if (dv.exp_buf && (threadIdx.x & 31) == 0 && blockIdx.x * 4 + threadIdx.x / 32 < 256) {
      const unsigned long long tx = globaltimer_ns();
      dv.exp_buf[dv.exp_slots + 8 + blockIdx.x * 4 + threadIdx.x / 32] = tx;
      atomicMax(dv.exp_buf + dv.exp_slots + 264 + (*(volatile uint32_t*)&dv.ctl->epoch % 64) * 4 + 2, tx);
    }
#endif
    return;
  }
  const uint32_t nside = (uint32_t)(qa.nfetch + qa.nfwd);
  const uint32_t bid = blockIdx.x - nside, nbid = gridDim.x - nside;  // lookup CTAs
  if (qa.dcnt && threadIdx.x == 0) {
    // key-sharded, sync-free: segment i's count is C[i][me] of the routed-count matrix in
    // device memory (written by the collective the stream ran before this launch)
    int64_t acc = 0;
    for (int i = 0; i < qa.n; ++i) {
      s_scan[i] = acc;
      acc += qa.dcnt[(size_t)i * qa.n + qa.dme];
    }
    s_scan[qa.n] = acc;
  }
#ifdef FLECHE_EXPERIMENTS
  if (dv.exp_buf && bid == 0 && threadIdx.x == 0) {
    const unsigned long long tx = globaltimer_ns();
    dv.exp_buf[dv.exp_slots + 1] = tx;
    dv.exp_buf[dv.exp_slots + 264 + (*(volatile uint32_t*)&dv.ctl->epoch % 64) * 4 + 0] = tx;
    dv.exp_buf[dv.exp_slots + 264 + (*(volatile uint32_t*)&dv.ctl->epoch % 64) * 4 + 2] = 0;
  }
#endif
  if (dv.ha && bid == 0 && threadIdx.x == 0)  // the host threads start streaming this batch's requests
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(dv.ha_start),
                 "l"((unsigned long long)*(volatile uint32_t*)&dv.ctl->epoch)
                 : "memory");
  __syncthreads();

  const int lane = threadIdx.x & 31;
  const int64_t N = s_scan[qa.n];
  uint32_t it = 0;  // grid-stride iterations (one unless the grid was sized for a capacity, not N)
  for (int64_t g0 = (int64_t)bid * blockDim.x; g0 < N; g0 += (int64_t)nbid * blockDim.x, ++it) {
  const int64_t g = g0 + threadIdx.x;
  if (g - lane < N) {  // warp-uniform
    const uint32_t epoch = *(volatile uint32_t*)&dv.ctl->epoch;
    const bool active = g < N;

    // A1 self-identification: largest t with scan[t] <= g (reading R14)
    int t = 0;
    int64_t j = 0, id = -1;
    if (!qa.fkeys) {
      if (active) {
        int lo = 0, hi = qa.n;
        while (hi - lo > 1) {
          const int mid = (lo + hi) >> 1;
          if (s_scan[mid] <= g) lo = mid; else hi = mid;
        }
        t = lo;
      }
      j = g - s_scan[t];
      if (active) id = qa.ids[t][j];
    } else if (active) {
      // key-sharded owner side: lookups arrive as flat keys; decode the table by prefix
      // match (largest base <= fk, the canonical size-aware code) and id = fk - base_t
      uint32_t fk0;
      if (qa.fkseg) {  // fused exchange: one segment per source rank (ids[] hold the segment pointers)
        int a = 0, b2 = qa.n;
        while (b2 - a > 1) {
          const int mid = (a + b2) >> 1;
          if (s_scan[mid] <= g) a = mid; else b2 = mid;
        }
        fk0 = ((const uint32_t*)qa.ids[a])[g - s_scan[a]];
      } else {
        fk0 = qa.fkeys[g];
      }
      int lo = 0, hi = dv.ntables;
      while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if ((uint32_t)(dv.kdec[mid] >> 16) <= fk0) lo = mid; else hi = mid;
      }
      t = (int)(dv.kdec[lo] & 0xFFFFu);
      id = (int64_t)(fk0 - (uint32_t)(dv.kdec[lo] >> 16));
      j = g;
    }
    const TableInfo* ti = dv.tables + qa.t0 + t;
    const int64_t card = ti->card;
    const int d = ti->dim;

    // A2 re-encode to the flat key (size-aware code: fk = base_t + id)
    const bool valid = active && id >= 0 && id < card;
    if (valid && ti->hashed && !qa.fkeys) id = short_feature_id(qa.t0 + t, id, ti->hmask);  // R24
    const uint32_t fk = valid ? ti->base + (uint32_t)id : kEmpty;
    const uint32_t s = valid ? set_of_t(dv, ti, fk) : 0u;

    // in-warp key groups (Zipf batches repeat hot keys within a warp): the lowest lane of
    // each group (its first occurrence) probes, refreshes the timestamp and claims the
    // miss for the whole group; the others take its result
    const unsigned peers = __match_any_sync(kFull, fk);
    const int klead = __ffs(peers) - 1;
    const bool lead = lane == klead;
    const unsigned pm = __ballot_sync(kFull, valid && lead);  // lanes whose set line is read

    // A3 probe: lane k holds way k of each probed set (one 128 B line each)
    // (FL_KQ_PROBE lines in flight per lane: fewer registers, more CTAs per SM)
    int way = -1;
#pragma unroll
    for (int i0 = 0; i0 < 32; i0 += FL_KQ_PROBE) {
      uint32_t kw[FL_KQ_PROBE];
#pragma unroll
      for (int i = 0; i < FL_KQ_PROBE; ++i) {
        const uint32_t si = __shfl_sync(kFull, s, i0 + i);
        kw[i] = ((pm >> (i0 + i)) & 1u) ? ld_nc_u32(dv.keys + (size_t)si * 32u + lane) : kEmpty;
      }
#pragma unroll
      for (int i = 0; i < FL_KQ_PROBE; ++i) {
        const uint32_t fki = __shfl_sync(kFull, fk, i0 + i);
        const unsigned m = __ballot_sync(kFull, kw[i] == fki);
        if (lane == i0 + i && m) way = __ffs(m) - 1;
      }
    }
    way = __shfl_sync(kFull, way, klead);
    const bool hit = valid && way >= 0;
    const bool miss = valid && way < 0;
    const uint32_t slot = s * 32u + (uint32_t)way;
    const int64_t off = active ? qa.out_off[t] + j * (int64_t)d : 0;

    // A4 hit gather from the HBM slab (zero row for an invalid ID); misses are KM's
    const float* src = nullptr;
    if (hit) {
      if (!dv.bytes) {
        src = slot_row(dv, ti, slot, d);
      } else {
        const uint32_t l = ld_nc_u32((const uint32_t*)(dv.loc + (slot & ~1u))) >> ((slot & 1u) * 16);
        src = dv.slab + ((size_t)s * dv.set_units + (l & 0xFFu)) * 8u;
      }
    }
    float* dst = (active && !miss) ? qa.out + off : nullptr;
    // issue the timestamp read (hits) and the first scratch read (misses) now, so their
    // L2 round trips overlap the row gather; they are consumed after it
    uint32_t old_ts = 0, h = 0;
    unsigned long long cur = 0;
    if (hit && lead) old_ts = ld_cg_u32(dv.ts + slot);
    if (miss && lead) {
      h = dv.ordered ? (uint32_t)__umul64hi((uint64_t)(ti->host + (size_t)id * (size_t)d) - dv.host_lo, dv.host_mul) &
                           dv.scr_mask
                     : scr_hash(fk) & dv.scr_mask;
      cur = ld_cg_u64(dv.scratch + h);
    }
    float* wsm = nullptr;
    if constexpr (TD > 0) wsm = kq_dyn + (size_t)(threadIdx.x >> 5) * 32 * TD;
    const unsigned mb = TD > 0 ? (unsigned)__cvta_generic_to_shared(&s_mbar[threadIdx.x >> 5]) : 0u;
    if (!qa.slots) {
      if constexpr (TD > 0) {
        // hit rows -> this warp's shared-memory block by bulk copies (no registers held while
        // they fly; the timestamp and dedup atomics below overlap them); invalid IDs -> zero
        // rows; miss rows are left for KM, which writes them after this grid
        const unsigned hm0 = __ballot_sync(kFull, hit);
        if (lane == 0) mbar_expect_tx(mb, (unsigned)__popc(hm0) * 4u * TD);
        __syncwarp();
        if (hit) bulk_g2s(wsm + lane * TD, src, 4u * TD, mb);
        if (active && !valid) {
#pragma unroll
          for (int c = 0; c < TD / 4; ++c) reinterpret_cast<float4*>(wsm + lane * TD)[c] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
      } else {
        gather_dispatch(src, dst, d, active, lane);
      }
    } else if (active) {  // decoupled: KG copies the hits on a side stream while KM fetches misses
      qa.slots[g] = hit ? slot : (miss ? kSlotMiss : kSlotZero);
    }

    // hit: refresh the way's timestamp once per batch (approximate LRU)
#if FL_KQ_TS_DEFER
    // issued predicated (no branch) and consumed only at the stats ballot, so its L2 round
    // trip overlaps the miss lanes' dedup CAS instead of preceding it
    const uint32_t need = (hit && lead && old_ts != epoch) ? 1u : 0u;
    uint32_t prev_ts = epoch;
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p atom.global.exch.b32 %0, [%1], %3;\n\t}"
                 : "+r"(prev_ts) : "l"(dv.ts + slot), "r"(need), "r"(epoch) : "memory");
#else
    bool uhit = false;
    if (hit && lead && old_ts != epoch) uhit = atomicExch(dv.ts + slot, epoch) != epoch;
#endif

    // A5 miss dedup: the lane whose CAS installs (epoch, fk) owns the miss
    int kind = 0;  // 1 = owner, 2 = duplicate
    uint32_t scr = 0;
    if (miss && lead) {
      const unsigned long long tag = ((unsigned long long)epoch << 32) | fk;
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
      // first occurrence of the key in canonical (table-major) order: the insert priority
      atomicMin(dv.firstpos + h, ((unsigned long long)(~epoch) << 32) | (uint32_t)(qa.g0 + g));
    }
    {  // the group's later lanes are duplicates of its leader's key
      const uint32_t scr_l = __shfl_sync(kFull, scr, klead);
      if (miss && !lead) {
        kind = 2;
        scr = scr_l;
      }
    }

    const int par = epoch & 1u;
    const unsigned own_m = __ballot_sync(kFull, kind == 1);
    const unsigned dup_m = __ballot_sync(kFull, kind == 2);
    const unsigned lt = (1u << lane) - 1u;
    if (own_m) {  // append to this width's region of the miss list, aggregated per class
      const int cls = ti->cls;
      const unsigned grp = __match_any_sync(kFull, kind == 1 ? cls : 64 + lane);
      const int leader = __ffs(grp) - 1;
      uint32_t b = 0;
      if (kind == 1 && lane == leader) b = atomicAdd(&dv.ctl->counts[par][cls], (uint32_t)__popc(grp));
      b = __shfl_sync(kFull, b, leader);
      uint64_t hst = kNoStage;
      if (kind == 1) {
        const uint32_t r = b + __popc(grp & lt);  // the miss's index within its width class
        const int64_t li = qa.cls_off[cls] + r;    // miss-list index
        // host-assisted: staging row ha_rbase[cls] + r (one request slot each); a class's
        // misses past its ha_rcap rows are read zero-copy (see ha_hcut for the ownership)
        const bool staged = dv.ha && r < dv.ha_rcap[cls];
        const uint32_t srow = staged ? dv.ha_rbase[cls] + r : 0u;
        if (staged) hst = (uint64_t)srow * dv.ha_row_floats;
        dv.miss[li] = MissRec{off, fk, scr, qa.t0 + t, 0, hst};
        dv.owner_off[scr] = off;
#ifdef FLECHE_EXPERIMENTS
        if (dv.exp_mode != 4)
#endif
        if (staged)  // the host threads' request, tagged with the epoch (no fence needed)
        {
          const HaReq rq = ha_req_make(qa.t0 + t, id, hst, epoch);
          if (qa.nfwd)  // to HBM; KQ's forwarder CTAs move it to the host in 1 KiB blocks
            asm volatile("st.global.cg.v2.u64 [%0], {%1, %2};" ::"l"(dv.ha_reqd + srow), "l"(rq.tid), "l"(rq.stage)
                         : "memory");
          else
            asm volatile("st.global.v2.u64 [%0], {%1, %2};" ::"l"(dv.ha_req + (size_t)par * dv.ha_req_cap + srow),
                         "l"(rq.tid), "l"(rq.stage)
                         : "memory");
        }
      }
    }
    if (dup_m) {
      uint32_t b = 0;
      if (lane == __ffs(dup_m) - 1) b = atomicAdd(&dv.ctl->counts[par][kDupSlot], (uint32_t)__popc(dup_m));
      b = __shfl_sync(kFull, b, __ffs(dup_m) - 1);
      if (kind == 2) dv.dup[b + __popc(dup_m & lt)] = DupRec{off, scr, d};  // restored by KD
    }

    if (qa.hit_flags && active) qa.hit_flags[g] = hit ? 1 : 0;  // key-sharded: per-key hit back to requester

    // A9 stats, warp-aggregated, straight into a striped counter row (fire-and-forget
    // reductions: no block barrier, so a finished warp retires without waiting for the
    // slowest warp of its CTA)
    const unsigned hm = __ballot_sync(kFull, hit), mm = __ballot_sync(kFull, miss);
#if FL_KQ_TS_DEFER
    const bool uhit = need && prev_ts != epoch;
#endif
    const unsigned im = __ballot_sync(kFull, active && !valid), um = __ballot_sync(kFull, uhit);
    if (lane == 0) {
      unsigned long long* row = dv.stats + ((blockIdx.x * 4u + (threadIdx.x >> 5)) % kStripes) * kNumCtr;
      if (hm) atomicAdd(row + C_HITS, (unsigned long long)__popc(hm));
      if (mm) atomicAdd(row + C_MISSES, (unsigned long long)__popc(mm));
      if (im) {
        atomicAdd(row + C_INVALID, (unsigned long long)__popc(im));
        dv.ctl->err_invalid = 1u;
      }
      if (um) atomicAdd(row + C_UHITS, (unsigned long long)__popc(um));
      if (own_m) atomicAdd(row + C_UMISS, (unsigned long long)__popc(own_m));
      if (dup_m) atomicAdd(row + C_DUPS, (unsigned long long)__popc(dup_m));
    }
    if constexpr (TD > 0) {
      if (!qa.slots) {  // the rows have landed: the warp's output rows leave as one contiguous block
        mbar_wait(mb, it & 1u);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // the zero rows, for the bulk store
        __syncwarp();
        const unsigned na = (unsigned)__popc(__ballot_sync(kFull, active));  // a prefix of the warp
        if (lane == 0) {
          bulk_s2g(qa.out + off, wsm, na * 4u * TD);  // lane 0's row starts the block (uniform rows)
          asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
        }
        __syncwarp();
      }
    }
  }
  }  // grid-stride loop
  if (qa.ha_bell) {
    // host-assisted fetch: the last CTA to finish rings the doorbell once every CTA has
    // counted its misses (earlier than KM could).  No system fence: the requests carry
    // epoch tags and the host threads wait for them (ha_req_current); no fence before the
    // arrival either: the warps' miss-count atomics returned their values, so they are
    // performed (a fence would also wait for the request stores to cross the link).
    // (Per-warp arrivals instead of this CTA barrier measured slower: one L2 atomic per
    // warp on one address, cfg2 KQ 46 vs 39 us, cfg5 268 vs 208 us, profiles/r02b/wb_*.)
    __syncthreads();
    if (threadIdx.x == 0) {
      const uint32_t prev = atomicAdd(&dv.ctl->kq_done, 1u);
      if (prev == nbid - 1) {
        __threadfence();
        dv.ctl->kq_done = 0;
        const uint32_t epoch = *(volatile uint32_t*)&dv.ctl->epoch;
        const int par = epoch & 1u;
        uint32_t cnt[8], total = 0;
        for (int c = 0; c < 8; ++c) {
          cnt[c] = c < qa.ncls ? *(volatile uint32_t*)&dv.ctl->counts[par][c] : 0u;
          total += cnt[c];
        }
        const uint32_t frac = *(volatile uint32_t*)&dv.ctl->ha_frac_q16;  // KM reads the same value
        if (frac && total >= dv.ha_min_rows) {  // KM's ha_active() takes the same decision
          HaDesc hd;
          hd.epoch = epoch;
          for (int c = 0; c < 8; ++c) {
            hd.cnt[c] = cnt[c];
            hd.hcut[c] = c < qa.ncls ? ha_hcut(cnt[c], dv.ha_rcap[c], frac) : 0u;
          }
          hd.pad = 0;
          hd.epoch2 = epoch;
          dv.ha_desc[par] = hd;  // no system fence: the host re-reads until both epoch fields match
          asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(dv.ha_bell), "l"((unsigned long long)epoch) : "memory");
          *(volatile uint32_t*)&dv.ctl->ha_rung = epoch;
        }
        if (nside) st_release_gpu_u32(&dv.ctl->kq_end, epoch);  // the fetch / forward CTAs: counts are final
#ifdef FLECHE_EXPERIMENTS
        if (dv.exp_buf) {
          dv.exp_buf[dv.exp_slots + 2] = globaltimer_ns();
          dv.exp_buf[dv.exp_slots + 264 + (epoch % 64) * 4 + 1] = dv.exp_buf[dv.exp_slots + 2];
        }
#endif
      }
    }
  }
  pdl_trigger();  // KM may be scheduled now; its pdl_wait still waits for this grid
}

// KG decoupled hit copy (Fig 8b): KQ only indexes (slot per lookup); KG copies
// the hit rows from the slab on a side stream WHILE KM fetches the misses over the host
// link -- the copy leaves the critical path of the miss handling.
template <int MAXT>
__global__ void __launch_bounds__(128) kg_kernel(const __grid_constant__ QArgs<MAXT> qa, const __grid_constant__ Dev dv) {
  __shared__ int64_t s_scan[MAXT + 1];
  for (int i = threadIdx.x; i <= qa.n; i += blockDim.x) s_scan[i] = qa.scan[i];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t N = s_scan[qa.n];
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g - lane >= N) return;
  const bool active = g < N;
  int t = 0;
  if (active) {
    int lo = 0, hi = qa.n;
    while (hi - lo > 1) {
      const int mid = (lo + hi) >> 1;
      if (s_scan[mid] <= g) lo = mid; else hi = mid;
    }
    t = lo;
  }
  const TableInfo* ti = dv.tables + t;
  const int d = ti->dim;
  const uint32_t code = active ? qa.slots[g] : kSlotMiss;
  const float* src = nullptr;
  float* dst = nullptr;
  if (code != kSlotMiss) {
    dst = qa.out + qa.out_off[t] + (g - s_scan[t]) * (int64_t)d;
    if (code != kSlotZero) {
      if (!dv.bytes) {
        src = slot_row(dv, ti, code, d);
      } else {
        const uint32_t l = ld_nc_u32((const uint32_t*)(dv.loc + (code & ~1u))) >> ((code & 1u) * 16);
        src = dv.slab + ((size_t)(code >> 5) * dv.set_units + (l & 0xFFu)) * 8u;
      }
    }
  }
  gather_dispatch(src, dst, d, active, lane);
}

// Uniform layout: claim a way for fk (first occurrence `pos` in the batch).
//  * victim = argmin (ts, key) over ways not read or written in this batch, claimed by a
//    CAS on its insert word ipos (epoch << 32 | pos << 1 | BUSY), then ts := epoch;
//  * no such way left: take over the way inserted in this batch by the miss with the
//    LARGEST first-occurrence position, if that is larger than ours.
// The set then ends up holding exactly the set's earliest-occurring misses, with exactly
// the argmin-(ts, key) candidates evicted -- what the oracle's first-occurrence insert
// order produces (reading R7) -- whatever order the warps run in.
// Returns the slot (>= 0), kClaimBypass, or kClaimRetry (the way to take over is still
// being written by its claimer: try again after this warp's own writes).  One lane.
constexpr int64_t kClaimBypass = -1, kClaimRetry = -2;
__device__ __forceinline__ int64_t claim_victim(const Dev& dv, const TableInfo* ti, uint32_t fk, uint32_t epoch,
                                                uint32_t pos, uint32_t* old_key, bool* took_over) {
  const uint32_t s = set_of_t(dv, ti, fk);
  const int nways = ways_in_t(dv, ti, s);
  if (nways <= 0) return kClaimBypass;
  const uint32_t* kp = dv.keys + (size_t)s * 32u;
  uint32_t* tp = dv.ts + (size_t)s * 32u;
  unsigned long long* ip = dv.ipos + (size_t)s * 32u;
  const unsigned long long mine = ((unsigned long long)epoch << 32) | ((unsigned long long)pos << 1) | 1ull;
  while (true) {
    // argmin (ts, key) over the ways not touched in this batch; the 32 keys and stamps
    // arrive as 16 B vectors and are scanned with compile-time indices (no local memory)
    unsigned long long best = ~0ull;
    int bw = -1;
    uint32_t bkey = kEmpty;
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint4 a = ld_cg_v4u(kp + 4 * q), b = ld_cg_v4u(tp + 4 * q);
      const uint32_t ka[4] = {a.x, a.y, a.z, a.w}, ta[4] = {b.x, b.y, b.z, b.w};
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int w = 4 * q + j;
        const unsigned long long r = ((unsigned long long)ta[j] << 32) | ka[j];
        if (w < nways && ta[j] < epoch && r < best) { best = r; bw = w; bkey = ka[j]; }
      }
    }
    if (bw >= 0) {
      const unsigned long long cur = ld_cg_u64(ip + bw);
      if ((uint32_t)(cur >> 32) == epoch) continue;  // claimed an instant ago; its ts is on the way
      if (atomicCAS(ip + bw, cur, mine) != cur) continue;
      tp[bw] = epoch;
      *old_key = bkey;
      *took_over = false;
      return (int64_t)s * 32 + bw;
    }
    // every way was read or written in this batch: the latest-occurring insert of this
    // batch gives way if we occur earlier
    unsigned long long worst = 0;
    int ww = -1;
    for (int w = 0; w < nways; ++w) {
      const unsigned long long v = ld_cg_u64(ip + w);
      if ((uint32_t)(v >> 32) == epoch && (v | 1ull) > (worst | 1ull)) { worst = v; ww = w; }
    }
    if (ww < 0 || ((worst >> 1) & 0x7FFFFFFFull) <= pos) return kClaimBypass;
    if (worst & 1ull) return kClaimRetry;  // still being written by its claimer
    if (atomicCAS(ip + ww, worst, mine) != worst) continue;
    *old_key = ld_cg_u32(kp + ww);  // published before its claimer cleared BUSY (fenced)
    *took_over = true;
    return (int64_t)s * 32 + ww;
  }
}

// Bytes layout: warp-cooperative insert of one row (units x 32 B, staged in smem)
// into fk's set under the set's lock.  Evicts argmin (ts, key) among rows not touched
// in this batch until a way is free and the row fits the set's byte budget; places it
// first-fit, compacting the set's region through `cbuf` (set_units * 2 float4 of
// smem) when free space is fragmented.  Returns false (bypass) if no candidate is
// left; evictions already made stay made (as in the oracle's MODE_SETBYTES).
static __device__ bool bytes_insert(const Dev& dv, uint32_t fk, int units, const float4* row, uint32_t epoch, int lane,
                             unsigned& ev, long long& docc, float4* cbuf) {
  const uint32_t s = set_of(dv, fk);
  const int SU = (int)dv.set_units;
  uint32_t* lk = dv.lock + s;
  if (lane == 0) {
    while (atomicCAS(lk, 0u, 1u) != 0u) __nanosleep(32);
  }
  __syncwarp();
  __threadfence();
  uint32_t* kp = dv.keys + (size_t)s * 32u + lane;
  uint32_t* tp = dv.ts + (size_t)s * 32u + lane;
  uint16_t* lp = dv.loc + (size_t)s * 32u + lane;
  uint32_t k = ld_cg_u32(kp);
  const uint32_t t = ld_cg_u32(tp);
  uint32_t l = ld_cg_u16(lp);
  bool live = k != kEmpty;
  int my_sz = live ? (int)(l >> 8) : 0;
  int used = __reduce_add_sync(kFull, (unsigned)my_sz);
  bool ok = true;
  while (true) {
    const int nlive = __popc(__ballot_sync(kFull, live));
    if (nlive < 32 && used + units <= SU) break;
    const unsigned long long rank = (live && t < epoch) ? (((unsigned long long)t << 32) | k) : ~0ull;
    const unsigned long long best = warp_min_u64(rank);
    if (best == ~0ull) { ok = false; break; }
    const int v = __ffs(__ballot_sync(kFull, rank == best)) - 1;
    const int vsz = __shfl_sync(kFull, my_sz, v);
    used -= vsz;
    if (lane == 0) { ++ev; docc -= 32ll * vsz; }
    if (lane == v) { live = false; my_sz = 0; k = kEmpty; *kp = kEmpty; }
  }
  if (ok) {
    // occupancy bitmap of the region (SU <= 256 units -> 8 words)
    const int my_off = (int)(l & 0xFFu);
    uint32_t words[8];
#pragma unroll
    for (int w = 0; w < 8; ++w) {
      uint32_t mine = 0;
      if (live) {
        const int lo = max(my_off, 32 * w), hi = min(my_off + my_sz, 32 * w + 32);
        if (hi > lo) mine = (hi - lo == 32) ? kFull : (((1u << (hi - lo)) - 1u) << (lo - 32 * w));
      }
      words[w] = __reduce_or_sync(kFull, mine);
    }
    // first fit at an offset aligned to the row's size (row sizes are powers of two in
    // 32 B units): aligned power-of-two blocks keep the region from fragmenting, so the
    // compaction below is rarely needed (placement only; which rows are cached is unchanged)
    int start = -1;
    for (int base = 0; base < SU && start < 0; base += 32) {
      const int p = base + lane;
      bool fits = p + units <= SU && (p & (units - 1)) == 0;
      for (int u = 0; u < units && fits; ++u) fits = !((words[(p + u) >> 5] >> ((p + u) & 31)) & 1u);
      const unsigned b = __ballot_sync(kFull, fits);
      if (b) start = base + __ffs(b) - 1;
    }
    if (start < 0) {  // fragmented: pack the live rows to the front through smem, largest first
      float* region = dv.slab + (size_t)s * SU * 8u;
      for (int c = lane; c < SU * 2; c += 32) cbuf[c] = ld_cg_v4(region + 4 * c);
      __syncwarp();
      // new offset = bytes of the rows packed before mine: larger rows, then equal rows of
      // lower way (descending power-of-two sizes keep every row aligned)
      int new_off = 0;
      for (int w = 0; w < 32; ++w) {
        const int wsz = __shfl_sync(kFull, my_sz, w);
        if (wsz > my_sz || (wsz == my_sz && w < lane)) new_off += wsz;
      }
      for (int w = 0; w < 32; ++w) {
        const int wsz = __shfl_sync(kFull, my_sz, w);
        if (!wsz) continue;
        const int wo = __shfl_sync(kFull, my_off, w), wn = __shfl_sync(kFull, new_off, w);
        for (int c = lane; c < wsz * 2; c += 32) st_v4(region + (size_t)(wn * 2 + c) * 4, cbuf[wo * 2 + c]);
      }
      if (live) *lp = (uint16_t)((my_sz << 8) | new_off);
      const int aligned = (used + units - 1) & ~(units - 1);
      start = aligned + units <= SU ? aligned : used;
      __syncwarp();
    }
    float* dst = dv.slab + ((size_t)s * SU + start) * 8u;
    for (int c = lane; c < units * 2; c += 32) st_v4(dst + 4 * c, row[c]);
    const int fw = __ffs(~__ballot_sync(kFull, live)) - 1;
    if (lane == fw) {
      *kp = fk;
      *tp = epoch;
      *lp = (uint16_t)((units << 8) | start);
    }
    if (lane == 0) docc += 32ll * units;
  }
  __syncwarp();
  __threadfence();
  if (lane == 0) atomicExch(lk, 0u);
  __syncwarp();
  return ok;
}

// Host-assisted KM for row width D (FLECHE_FLAG_HOST_ASSIST): warp gw takes whole
// staging blocks (kHaBlock miss-list indices); lane 0 waits once for the block's ready
// flag, then the warp pulls all of the block's rows over the host link at once
// (ld.cv 16 B loads, 16 in flight per lane, into shared memory: two link round
// trips per block instead of one per chunk) -- staged rows from the contiguous staging
// buffer, rows without a staging slot (or after a timeout) from the tables -- and
// places them 32 at a time (one row per lane: admission, victim claim, slab + out).
template <bool BYTES, int D>
__device__ __forceinline__ void km_ha(const Dev& dv, float* __restrict__ out, const MissRec* __restrict__ mlist,
                                      uint32_t epoch, uint32_t nmiss, int lane, uint32_t gw, uint32_t nw, unsigned& ins,
                                      unsigned& ev, unsigned& byp, long long& docc, unsigned long long& hostb,
                                      float4* hsm, float4* cbuf, unsigned& harows, unsigned& hato, int cls,
                                      uint32_t hcut) {
  constexpr int VEC = D / 4;
  constexpr int ROWS0 = (kHaSmemF4 / VEC) < kHaBlock ? (kHaSmemF4 / VEC) : kHaBlock;  // rows that fit the warp's smem
  constexpr int ROWS = ROWS0 < 16 ? ROWS0 : 16;  // rows per piece: one warp per piece, pieces of a block in parallel
  constexpr int PPB = kHaBlock / ROWS;           // pieces per staging block
  constexpr int PER_LANE = ROWS * VEC / 32;      // float4 per lane per piece
  constexpr int INFL = PER_LANE < 16 ? PER_LANE : 16;
  const float* stage = dv.ha_stage + (size_t)(epoch & 1u) * dv.ha_stage_floats;
  const float* hstage = dv.ha_hstage ? dv.ha_hstage + (size_t)(epoch & 1u) * dv.ha_stage_floats : nullptr;
  // work unit = pieces of this class's miss list (class-local index j; a piece never
  // straddles a 64-row staging block): a staged piece starts as soon as its block is
  // ready, and the zero-copy pieces (blocks >= hcut, or past the class's staging rows) get
  // the whole grid's memory-level parallelism, not one warp per 64 rows.  Pieces per
  // unit: as fine as the grid allows (one piece per warp while there are enough warps,
  // cfg2 +8 %), coarser for big batches (cfg5 +8 %); FLECHE_HA_UNIT_PIECES fixes it (A/B)
  const uint32_t npieces = (nmiss + ROWS - 1) / ROWS;
  const uint32_t ppu = dv.ha_unit_pieces ? min((uint32_t)PPB, dv.ha_unit_pieces)
                                         : min((uint32_t)PPB, max(1u, (npieces + nw - 1) / nw));
  const uint32_t rcap = dv.ha_rcap[cls], blk0 = dv.ha_rbase[cls] / kHaBlock;
  for (uint32_t u0 = gw * ppu; u0 < npieces; u0 += nw * ppu)
  for (uint32_t u = u0; u < min(u0 + ppu, npieces); ++u) {
    const uint32_t blo = u * ROWS, bhi = min(blo + (uint32_t)ROWS, nmiss);
    const uint32_t hb = blo / kHaBlock, pc = (blo % kHaBlock) / ROWS;  // class-local staging block
    const uint32_t kb = blk0 + hb;                                     // its absolute block id
    int ok = 0;
#ifdef FLECHE_EXPERIMENTS
    if (dv.exp_blk && lane == 0 && pc == 0) dv.exp_blk[kb * 8 + 0] = globaltimer_ns();
#endif
    if (lane == 0 && blo < rcap && hb < hcut) {  // the host threads' share; the rest from the tables
      if (dv.ha_hstage && ld_acquire_gpu_u32(dv.ha_hseen + kb) == epoch) {
        ok = 2;  // early fetch already moved the block into HBM
      } else {
        ok = ha_wait_block(dv, epoch, kb);
        if (!ok && pc == 0) ++hato;
      }
    }
#ifdef FLECHE_EXPERIMENTS
    if (dv.exp_blk && lane == 0 && pc == 0) dv.exp_blk[kb * 8 + 1] = globaltimer_ns();
#endif
    ok = __shfl_sync(kFull, ok, 0);
    for (uint32_t plo = blo; plo < bhi; plo += ROWS) {  // one iteration: the piece
      const uint32_t n = min((uint32_t)ROWS, bhi - plo);
      // the piece's miss records (row r on lane r % 32) and row sources
      MissRec m[(ROWS + 31) / 32];
      const float* src[(ROWS + 31) / 32];
#pragma unroll
      for (int h = 0; h < (ROWS + 31) / 32; ++h) {
        const uint32_t r = h * 32 + lane;
        src[h] = nullptr;
        if (r < n) {
          m[h] = mlist[plo + r];
          const TableInfo* ti = dv.tables + m[h].t;
          const bool st = ok && m[h].hst != kNoStage;
          src[h] = st ? (ok == 2 ? hstage : stage) + m[h].hst : ti->host + (size_t)(m[h].fk - ti->base) * D;
          if (st) ++harows;
          hostb += 4ull * D;
        }
      }
      // all rows of the piece over the link into shared memory
#pragma unroll 1
      for (int q0 = 0; q0 < PER_LANE; q0 += INFL) {
        float4 v[INFL];
#pragma unroll
        for (int i = 0; i < INFL; ++i) {
          const int q = (q0 + i) * 32 + lane, r = q / VEC, c = q % VEC;
          const float* s0 = (const float*)__shfl_sync(kFull, (unsigned long long)src[0], r & 31);
          const float* s1 = (ROWS > 32) ? (const float*)__shfl_sync(kFull, (unsigned long long)src[(ROWS + 31) / 32 - 1], r & 31)
                                        : s0;
          const float* sp = r < 32 ? s0 : s1;
          v[i] = (r < (int)n && sp) ? ld_cv_v4(sp + 4 * c) : make_float4(0.f, 0.f, 0.f, 0.f);
        }
#pragma unroll
        for (int i = 0; i < INFL; ++i) hsm[(q0 + i) * 32 + lane] = v[i];
      }
      __syncwarp();
#ifdef FLECHE_EXPERIMENTS
      if (dv.exp_blk && lane == 0 && plo == blo) dv.exp_blk[kb * 8 + 2] = globaltimer_ns();
#endif
      // place the rows, 32 at a time (lane = row)
#pragma unroll
      for (int h = 0; h < (ROWS + 31) / 32; ++h) {
        const uint32_t r = h * 32 + lane;
        const bool has = r < n;
        const MissRec mm = has ? m[h] : MissRec{};
        const float* row = (const float*)(hsm + (size_t)r * VEC);
        bool admit = false;
        if (has)
          admit = dv.admit_all ||
                  splitmix64(dv.admit_seed ^ (uint64_t)mm.fk ^ ((uint64_t)(epoch - 1u) << 32)) < dv.admit_thr;
        if constexpr (!BYTES) {
          bool pending = has && admit;
          if (has && !admit) ++byp;
          const TableInfo* ti = dv.tables + (has ? mm.t : 0);
          const uint32_t pos = pending ? (uint32_t)ld_cg_u64(dv.firstpos + mm.scr) : 0u;
          while (__any_sync(kFull, pending)) {
            float* slab_dst = nullptr;
            int64_t slot = kClaimRetry;
            if (pending) {
              uint32_t old_key = kEmpty;
              bool took = false;
              slot = claim_victim(dv, ti, mm.fk, epoch, pos, &old_key, &took);
              if (slot >= 0) {
                pending = false;
                if (took) {
                  ++byp;
                } else {
                  ++ins;
                  docc += 4ll * D;
                  if (old_key != kEmpty) { ++ev; docc -= 4ll * D; }
                }
                slab_dst = slot_row(dv, ti, (uint32_t)slot, D);
              } else if (slot == kClaimBypass) {
                pending = false;
                ++byp;
              }
            }
            copy_rows_generic<D>(row, slab_dst, lane);
            if (slab_dst) {
              dv.keys[slot] = mm.fk;
              __threadfence();
              *(volatile unsigned long long*)(dv.ipos + slot) = ((unsigned long long)epoch << 32) | ((unsigned long long)pos << 1);
            }
            if (slot == kClaimRetry && pending) __nanosleep(100);
          }
        } else {
          for (int q = 0; q < 32; ++q) {  // inserts, one set lock at a time
            if (!__shfl_sync(kFull, (int)has, q)) continue;
            const uint32_t fk = __shfl_sync(kFull, mm.fk, q);
            if (!__shfl_sync(kFull, (int)admit, q)) {
              if (lane == 0) ++byp;
              continue;
            }
            const bool okk = bytes_insert(dv, fk, D / 8, hsm + (size_t)(h * 32 + q) * VEC, epoch, lane, ev, docc, cbuf);
            if (lane == 0) { if (okk) ++ins; else ++byp; }
          }
        }
        copy_rows_generic<D>(row, has ? out + mm.off : nullptr, lane);  // the owner's output row
      }
      __syncwarp();
    }
#ifdef FLECHE_EXPERIMENTS
    if (dv.exp_blk && lane == 0) dv.exp_blk[kb * 8 + 3] = globaltimer_ns();
#endif
  }
}

// KM for row width D: each warp iteration handles M unique misses of this class.
template <bool BYTES, int D, int M>
__device__ __forceinline__ void km_rows(const Dev& dv, float* __restrict__ out, const MissRec* __restrict__ mlist,
                                        uint32_t epoch, uint32_t nmiss, int lane, uint32_t gw, uint32_t nw,
                                        unsigned& ins, unsigned& ev, unsigned& byp, long long& docc,
                                        unsigned long long& hostb, float4* wsm) {
#ifdef FLECHE_EXPERIMENTS
  if (dv.exp_buf && lane == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    dv.exp_buf[gw * 4 + 0] = t;
    dv.exp_buf[gw * 4 + 1] = 0;
  }
#endif
  bool first_chunk = true;
  // one chunk of up to M unique misses (lane r < M holds miss r)
  auto chunk = [&](bool has, MissRec m) {
    const float* src = nullptr;
    if (has) {
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
    bool admit = false;
    if (has) {
      admit = dv.admit_all ||
              splitmix64(dv.admit_seed ^ (uint64_t)m.fk ^ ((uint64_t)(epoch - 1u) << 32)) < dv.admit_thr;
      hostb += 4ull * D;
    }
    if constexpr (!BYTES) {
      // A7 while the loads are in flight: victim claim (L2 round trips only); the first
      // use of the loaded rows (the slab store) comes after this round's claims
      bool pending = has && admit;
      if (has && !admit) ++byp;
      const TableInfo* ti = dv.tables + (has ? m.t : 0);
      const uint32_t pos = pending ? (uint32_t)ld_cg_u64(dv.firstpos + m.scr) : 0u;
      while (__any_sync(kFull, pending)) {  // rounds: a lane may wait for a way its warp still writes
        float* slab_dst = nullptr;
        int64_t slot = kClaimRetry;
        if (pending) {
          uint32_t old_key = kEmpty;
          bool took = false;
          slot = claim_victim(dv, ti, m.fk, epoch, pos, &old_key, &took);
          if (slot >= 0) {
            pending = false;
            if (took) {
              ++byp;  // the later-occurring miss we displaced is bypassed; our insert replaces its
            } else {
              ++ins;
              docc += 4ll * D;
              if (old_key != kEmpty) { ++ev; docc -= 4ll * D; }
            }
            slab_dst = slot_row(dv, ti, (uint32_t)slot, D);
          } else if (slot == kClaimBypass) {
            pending = false;
            ++byp;
          }
        }
        rb.store(slab_dst, lane);
        if (slab_dst) {  // row -> key -> release the way (clears BUSY)
          dv.keys[slot] = m.fk;
          __threadfence();
          *(volatile unsigned long long*)(dv.ipos + slot) = ((unsigned long long)epoch << 32) | ((unsigned long long)pos << 1);
        }
        if (slot == kClaimRetry && pending) __nanosleep(100);
      }
      rb.store(has ? out + m.off : nullptr, lane);  // the owner's output row
#ifdef FLECHE_EXPERIMENTS
      if (dv.exp_buf && lane == 0 && first_chunk) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        dv.exp_buf[gw * 4 + 1] = t;
        dv.exp_buf[gw * 4 + 3] = (unsigned long long)__popc(__activemask());
      }
#endif
    } else {
      rb.store(has ? out + m.off : nullptr, lane);
      rb.to_smem(wsm, lane);
      __syncwarp();
      for (int r = 0; r < M; ++r) {  // inserts of this chunk, one set lock at a time
        if (!__shfl_sync(kFull, (int)has, r)) continue;
        const uint32_t fk = __shfl_sync(kFull, m.fk, r);
        if (!__shfl_sync(kFull, (int)admit, r)) {
          if (lane == 0) ++byp;
          continue;
        }
        const bool ok = bytes_insert(dv, fk, D / 8, wsm + r * (D / 4), epoch, lane, ev, docc, wsm + kKmStageF4);
        if (lane == 0) { if (ok) ++ins; else ++byp; }
      }
    }
    __syncwarp();
    first_chunk = false;
  };

  if (BYTES || !dv.ordered) {  // misses from this width's region of the miss list
    for (uint32_t base = gw * M; base < nmiss; base += nw * M) {
      const uint32_t k = base + lane;
      const bool has = lane < M && k < nmiss;
      MissRec m{};
      if (has) m = mlist[k];
      chunk(has, m);
    }
  } else {
    // address-ordered scratch (slot ~ host address).  Band-major sweep: the slot space is cut
    // into B bands of about M misses per warp each, and band b is cut into nw sub-windows, so
    // round b of every warp reads rows of band b: the batch's host reads sweep the host tier
    // once in address order and the reads in flight at any time share a narrow address band
    // (translation locality: a sorted burst of 8K rows ran 92 vs 115 us unsorted,
    // profiles/burst_cold_r02.json).  dv.bands < 0: one contiguous window per warp.
    const uint32_t nslots = dv.scr_mask + 1u;
    const uint32_t bw = dv.bands > 0 ? (uint32_t)dv.bands : (uint32_t)M;  // misses per warp per band
    const uint32_t B = dv.bands >= 0 ? max(1u, (nmiss + nw * bw - 1) / (nw * bw)) : 1u;
    const uint32_t band = (nslots + B - 1) / B;
    const uint32_t per = (band + nw - 1) / nw;
    uint32_t my_slot = 0;
    int P = 0;  // misses collected so far (lanes 0..P-1 hold their slots)
    auto flush = [&]() {
      MissRec m{};
      const bool has = lane < P;
      if (has) {
        const unsigned long long tag = ld_cg_u64(dv.scratch + my_slot);
        m.fk = (uint32_t)tag;
        m.scr = my_slot;
        m.off = dv.owner_off[my_slot];
        int a = 0, b = dv.ntables;  // decode the table from the flat key (prefix match)
        while (b - a > 1) {
          const int mid = (a + b) >> 1;
          if ((uint32_t)(dv.kdec[mid] >> 16) <= m.fk) a = mid; else b = mid;
        }
        m.t = (int32_t)(dv.kdec[a] & 0xFFFFu);
      }
      chunk(has, m);
      P = 0;
    };
    for (uint32_t b = 0; b < B; ++b) {
    const uint32_t lo = min(nslots, b * band + gw * per), hi = min(min(nslots, (b + 1) * band), lo + per);
    for (uint32_t s1 = lo; s1 < hi; s1 += 256) {  // 8 tag loads per lane in flight, then in order
      unsigned long long tags[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const uint32_t slot = s1 + 32 * i + lane;
        tags[i] = slot < hi ? ld_cg_u64(dv.scratch + slot) : 0ull;
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const uint32_t slot = s1 + 32 * i + lane;
        unsigned found = __ballot_sync(kFull, slot < hi && (uint32_t)(tags[i] >> 32) == epoch);
        while (found) {
          const int f = __ffs(found) - 1;
          found &= found - 1;
          const uint32_t fs = __shfl_sync(kFull, slot, f);
          if (lane == P) my_slot = fs;
          if (++P == M) flush();
        }
      }
    }
    }
    if (__any_sync(kFull, P > 0)) flush();
  }
#ifdef FLECHE_EXPERIMENTS
  if (dv.exp_buf && lane == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    dv.exp_buf[gw * 4 + 2] = t;
  }
#endif
}

// Misses per KM warp iteration for a row width (the KM shape sweep was flat within
// noise, profiles/README.md; these keep the rows of one iteration in registers)
template <bool BYTES, int D>
struct KmM {
  static constexpr int value = D >= 256 ? 4 : (BYTES || D >= 64 ? 8 : 16);
};

// The paper's unified-index capacity loop: "We start with an empty unified
// index, and keep gradually increasing its capacity ... We pause increasing until the
// performance peak is reached.  If a significant performance decline is detected (which
// means that workload changes), we clear the unified index and repeat."  Here the unified
// index costs no HBM (computed host addresses, R11); what it trades against is the
// CPU-DRAM layer: every staging block the GPU fetches itself (zero-copy) is one the host
// threads do not gather.  So the tuned quantity is the unified index's share of a batch's
// blocks, 1 - ha_frac: it starts at 0 (the host threads take every block), grows by
// kTuneStep per window of kTuneWin batches while the miss kernel's time per unique miss
// improves, pauses one step back at the peak, and restarts from 0 when a paused window is
// kTuneDecline slower than the peak.  While paused it re-probes one step to either side every
// kTuneProbe windows and keeps a probe that is kTuneGain faster (a single greedy climb from 0
// stopped on one noisy window: cfg4 settled at 0.0 or 0.4 from run to run).  A window is 16
// batches, or fewer when they are slow (at least 2 batches and 2 ms of KM time), so slow
// configurations are tuned within a few hundred milliseconds too.  Run by KM's last CTA; it
// changes where rows are read from only, never a result.
constexpr uint32_t kTuneWin = 16;
constexpr unsigned long long kTuneWinNs = 2000000;
constexpr uint32_t kTuneStep = 6554;  // 0.1 of the blocks (x 2^-16)
constexpr double kTuneDecline = 1.15;
constexpr uint32_t kTuneProbe = 4;
constexpr double kTuneGain = 0.97;
__device__ __forceinline__ void ui_tune(const Dev& dv, uint32_t nmiss) {
  Ctl* c = dv.ctl;
  const unsigned long long t = globaltimer_ns() - c->km_t0;
  if (dv.ha_frac_fixed || nmiss < dv.ha_min_rows || t > 1000000000ull) return;
  c->win_ns += t;
  c->win_miss += nmiss;
  ++c->win_n;
  if (c->win_n < kTuneWin && (c->win_n < 2 || c->win_ns < kTuneWinNs)) return;
  const double cost = (double)c->win_ns / (double)max(1ull, c->win_miss);
  c->win_ns = c->win_miss = 0;
  c->win_n = 0;
  uint32_t f = c->ha_frac_q16;
  if (c->tune_phase == 0) {  // growing the unified-index share
    if (c->prev_cost == 0.0 || cost < c->prev_cost) {
      c->prev_cost = cost;
      if (f > kTuneStep) {
        f -= kTuneStep;
      } else {
        c->tune_phase = 1;  // the unified index has every block: that is the peak
      }
    } else {
      f = min(65536u, f + kTuneStep);  // one step back: the previous share was the peak
      c->tune_phase = 1;
    }
    c->tune_since = 0;
  } else if (c->tune_phase == 1) {  // paused at the peak
    if (cost > c->prev_cost * kTuneDecline) {  // the workload changed: clear and repeat
      f = 65536u;
      c->tune_phase = 0;
      c->prev_cost = 0.0;
    } else {
      c->prev_cost = cost;  // the peak's current cost
      if (++c->tune_since >= kTuneProbe) {  // probe one step to one side
        c->tune_since = 0;
        c->tune_dir = c->tune_dir > 0 ? -1 : 1;
        const int64_t g = (int64_t)f + (int64_t)c->tune_dir * kTuneStep;
        if (g >= (int64_t)kTuneStep && g <= 65536) {
          c->tune_best = f;
          f = (uint32_t)g;
          c->tune_phase = 2;
        }
      }
    }
  } else {  // one probe window
    if (cost < c->prev_cost * kTuneGain) c->prev_cost = cost;  // better: the probe is the new peak
    else f = c->tune_best;
    c->tune_phase = 1;
  }
  c->ha_frac_q16 = f;
}

// DU > 0: uniform layout of width DU (one class); DU = 0: every width class in turn.
template <bool BYTES, int DU>
__global__ void __launch_bounds__(128, 4) km_kernel(const __grid_constant__ Dev dv, const __grid_constant__ KMArgs ka) {
  __shared__ unsigned long long s_ctr[kNumCtr];
  extern __shared__ float4 s_dyn[];
  if (threadIdx.x < kNumCtr) s_ctr[threadIdx.x] = 0;
  __syncthreads();
  pdl_wait();  // KQ has completed: miss lists and owner rows are final
  const uint32_t epoch = *(volatile uint32_t*)&dv.ctl->epoch;
  const int par = epoch & 1u;
  const int lane = threadIdx.x & 31;
  if (dv.ha && blockIdx.x == 0 && threadIdx.x == 0) dv.ctl->km_t0 = globaltimer_ns();  // (ui_tune)
  const bool use_ha = ha_active(dv, ka, par);  // KQ's last CTA rang the doorbell (same test)
  const uint32_t frac = use_ha ? *(volatile uint32_t*)&dv.ctl->ha_frac_q16 : 0u;  // as KQ's bell saw it
  if (use_ha && ka.bell && blockIdx.x == 0 && threadIdx.x == 0) {
    // doorbell from KM (ctx option): KQ's request writes completed with its grid
    HaDesc hd;
    hd.epoch = epoch;
    for (int c = 0; c < 8; ++c) {
      hd.cnt[c] = c < ka.ncls ? *(volatile uint32_t*)&dv.ctl->counts[par][c] : 0u;
      hd.hcut[c] = c < ka.ncls ? ha_hcut(hd.cnt[c], dv.ha_rcap[c], frac) : 0u;
    }
    hd.pad = 0;
    hd.epoch2 = epoch;
    dv.ha_desc[par] = hd;
    __threadfence_system();
    st_release_sys_u64(dv.ha_bell, (unsigned long long)epoch);
    *(volatile uint32_t*)&dv.ctl->ha_rung = epoch;
  }
  // block-interleaved warp numbering: consecutive miss chunks land on different SMs,
  // so the host-link loads of a batch are spread over the whole GPU
  uint32_t gw = (threadIdx.x >> 5) * gridDim.x + blockIdx.x;
  uint32_t nw = (gridDim.x * blockDim.x) >> 5;
  // per warp: [kHaSmemF4 host-assisted rows][kKmSmemF4 bytes-layout staging + compaction]
  const int wsm_f4 = (dv.ha ? kHaSmemF4 : 0) + (BYTES ? kKmSmemF4 : 0);
  float4* hsm = s_dyn + (threadIdx.x >> 5) * wsm_f4;
  float4* wsm = hsm + (dv.ha ? kHaSmemF4 : 0);
  unsigned ins = 0, ev = 0, byp = 0, harows = 0, hato = 0;
  long long docc = 0;
  unsigned long long hostb = 0;
  bool poller = false;
  if (use_ha) {  // warp 0 of CTA 0 polls the host threads' progress; the other warps read blocks
    poller = gw == 0;
    if (poller) {
      HaBlocks hb;
      hb.ncls = ka.ncls;
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        const uint32_t cnt = c < ka.ncls ? *(volatile uint32_t*)&dv.ctl->counts[par][c] : 0u;
        hb.lo[c] = dv.ha_rbase[c] / kHaBlock;
        hb.n[c] = c < ka.ncls ? ha_hcut(cnt, dv.ha_rcap[c], frac) : 0u;
      }
      ha_poll(dv, epoch, hb, lane);
    }
    gw -= 1;
    nw -= 1;
  }
  for (int c = 0; c < ka.ncls && !poller; ++c) {
    const uint32_t nmiss = *(volatile uint32_t*)&dv.ctl->counts[par][c];
    if (!nmiss) continue;
    const MissRec* ml = dv.miss + ka.cls_off[c];
#define FL_KM(D)                                                                                              \
  if (use_ha)                                                                                                 \
    km_ha<BYTES, D>(dv, ka.out, ml, epoch, nmiss, lane, gw, nw, ins, ev, byp, docc, hostb, hsm, wsm, harows, hato, c,  \
                    ha_hcut(nmiss, dv.ha_rcap[c], frac));                                                   \
  else                                                                                                        \
    km_rows<BYTES, D, KmM<BYTES, D>::value>(dv, ka.out, ml, epoch, nmiss, lane, gw, nw, ins, ev, byp, docc, hostb, wsm)
    if constexpr (DU > 0) {
      FL_KM(DU);
    } else {
      switch (ka.cls_dim[c]) {  // fleche_create only admits these widths
        case 8: FL_KM(8); break;
        case 16: FL_KM(16); break;
        case 32: FL_KM(32); break;
        case 64: FL_KM(64); break;
        case 128: FL_KM(128); break;
        case 256: FL_KM(256); break;
        default: break;
      }
    }
#undef FL_KM
  }
  ins = __reduce_add_sync(kFull, ins);
  ev = __reduce_add_sync(kFull, ev);
  byp = __reduce_add_sync(kFull, byp);
  harows = __reduce_add_sync(kFull, harows);
  hato = __reduce_add_sync(kFull, hato);
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    hostb += __shfl_xor_sync(kFull, hostb, o);
    docc += __shfl_xor_sync(kFull, docc, o);
  }
  if (lane == 0) {
    if (ins) atomicAdd(&s_ctr[C_INSERTED], (unsigned long long)ins);
    if (ev) atomicAdd(&s_ctr[C_EVICTED], (unsigned long long)ev);
    if (byp) atomicAdd(&s_ctr[C_BYPASSED], (unsigned long long)byp);
    if (harows) atomicAdd(&s_ctr[C_HAROWS], (unsigned long long)harows);
    if (hato) atomicAdd(&s_ctr[C_HATIMEOUT], (unsigned long long)hato);
    if (hostb) atomicAdd(&s_ctr[C_HOSTBYTES], hostb);
    if (docc) atomicAdd((unsigned long long*)&dv.ctl->occ_bytes, (unsigned long long)docc);
  }
  __syncthreads();
  if (threadIdx.x < kNumCtr && s_ctr[threadIdx.x])
    atomicAdd(dv.stats + (blockIdx.x % kStripes) * kNumCtr + threadIdx.x, s_ctr[threadIdx.x]);

  // A8 restore, the former third kernel (KD) of a batch: every later
  // occurrence of a missed key copies its owner's row once every owner row is in `out`.
  // Grid barrier first (the launch is cooperative, so every CTA is resident); skipped by
  // every CTA alike when the batch has no duplicate misses (the count is final: KQ wrote it).
  const uint32_t ndup = *(volatile uint32_t*)&dv.ctl->counts[par][kDupSlot];
  if (ndup) {
    if (threadIdx.x == 0) {
      __threadfence();
      const uint32_t prev = atomicAdd(&dv.ctl->done, 1u);
      if (prev == gridDim.x - 1) {
        dv.ctl->done = 0;
        st_release_gpu_u32(&dv.ctl->km_bar, epoch);
      } else {
        while (ld_acquire_gpu_u32(&dv.ctl->km_bar) != epoch) __nanosleep(64);
      }
    }
    __syncthreads();
    for (uint32_t i = gw; i < ndup; i += nw) {  // owner rows were written by other SMs: read via L2
      const DupRec r = dv.dup[i];
      const float* src = ka.out + dv.owner_off[r.scr];
      for (int c = lane; c < r.dim / 4; c += 32) st_v4(ka.out + r.off + 4 * c, ld_cg_v4(src + 4 * c));
    }
  }
  pdl_trigger();
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const uint32_t prev = atomicAdd(&dv.ctl->done2, 1u);
    if (prev == gridDim.x - 1) {  // last CTA closes the batch: next batch's counters, epoch + 1
      if (dv.ha) {
        uint32_t nm = 0;
        for (int c = 0; c < ka.ncls; ++c) nm += *(volatile uint32_t*)&dv.ctl->counts[par][c];
        ui_tune(dv, nm);
      }
#pragma unroll
      for (int c = 0; c < 8; ++c) dv.ctl->counts[par ^ 1][c] = 0;
      dv.ctl->done2 = 0;
      __threadfence();
      *(volatile uint32_t*)&dv.ctl->epoch = epoch + 1u;
    }
  }
}

// Pooling: one thread per (bag, 4-float column); sums the bag's staged
// rows sequentially in bag order in fp32 (the oracle's order, so results are
// bit-identical for any values).  An empty bag gives a zero row.
template <int MAXT>
__global__ void __launch_bounds__(256) kp_kernel(const __grid_constant__ PArgs<MAXT> pa, const TableInfo* __restrict__ tables) {
  __shared__ int64_t s_scan[MAXT + 1];
  for (int i = threadIdx.x; i <= pa.n; i += blockDim.x) s_scan[i] = pa.cscan[i];
  __syncthreads();
  pdl_wait();
  pdl_trigger();
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g >= s_scan[pa.n]) return;
  int lo = 0, hi = pa.n;
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (s_scan[mid] <= g) lo = mid; else hi = mid;
  }
  const int t = lo;
  const int vec = tables[t].dim / 4;
  const int64_t local = g - s_scan[t];
  const int64_t bag = local / vec;
  const int c = (int)(local % vec);
  const int64_t k0 = pa.offs[t][bag], k1 = pa.offs[t][bag + 1];
  const float* st = pa.stage + pa.stage_off[t] + 4 * c;
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int64_t k = k0; k < k1; ++k) {
    const float4 x = *reinterpret_cast<const float4*>(st + k * 4 * vec);
    acc.x = __fadd_rn(acc.x, x.x);
    acc.y = __fadd_rn(acc.y, x.y);
    acc.z = __fadd_rn(acc.z, x.z);
    acc.w = __fadd_rn(acc.w, x.w);
  }
  *reinterpret_cast<float4*>(pa.out + pa.out_off[t] + bag * 4 * vec + 4 * c) = acc;
}

// Watermark (full-scan) eviction, the paper's replacement trigger: "when the
// utilization of the memory pool exceeds a certain threshold, FC performs cache eviction
// with a full table scan and keeps evicting cold embeddings until memory utilization
// falls below another threshold"; entries read in the current epoch are never reclaimed
// (epoch-based reclamation).  Reading R23: checked once per batch
// after its inserts; coldness = age class min(epoch - ts, kAgeBins - 1); whole classes
// are evicted, oldest first, until the cached row bytes are <= lo.  Two launches after
// KD: KE1 builds the byte histogram of age classes, KE2 picks the threshold class A (every
// CTA redundantly, from the 32 KB histogram in L2) and evicts every untouched way of age
// >= A.  Both exit at once when the bytes are <= hi, so an idle scan costs two launches.
constexpr int kAgeBins = 4096;  // ages saturate at 4095 batches (reading R23)

struct KEArgs {
  unsigned long long* hist;  // [kAgeBins] row bytes per age class (zero between scans)
  long long hi, lo;          // watermarks in row bytes
};

__device__ __forceinline__ uint32_t way_units(const Dev& dv, size_t i) {  // row bytes / 32
  return dv.bytes ? (uint32_t)(ld_cg_u16(dv.loc + i) >> 8) : (uint32_t)(dv.dim >> 3);
}

template <int = 0>
__global__ void __launch_bounds__(256) ke_hist_kernel(const __grid_constant__ Dev dv, const __grid_constant__ KEArgs ea) {
  __shared__ uint32_t h[kAgeBins];  // 32-byte units per age class
  for (int i = threadIdx.x; i < kAgeBins; i += blockDim.x) h[i] = 0;
  __syncthreads();
  pdl_wait();
  const uint32_t epoch = *(volatile uint32_t*)&dv.ctl->epoch - 1u;  // KM advanced it
  // nothing changes occ_bytes while KE1 runs (KM has completed, KE2 has not started), so
  // every CTA reads the same value; CTA 0 records it as the scan's one snapshot for KE2,
  // whose CTAs lower occ_bytes while others may not have started yet
  const long long occ = *(volatile long long*)&dv.ctl->occ_bytes;
  if (blockIdx.x == 0 && threadIdx.x == 0) dv.ctl->ke_occ = occ;
  if (occ <= ea.hi) {
    pdl_trigger();
    return;
  }
  const size_t quads = (size_t)dv.sets * 8u;  // 4 ways per thread step (16 B of keys + ts)
  const size_t qend = (quads + 31) & ~(size_t)31;  // whole warps stay in the loop (match below)
  const int lane = threadIdx.x & 31;
  for (size_t q = (size_t)blockIdx.x * blockDim.x + threadIdx.x; q < qend; q += (size_t)gridDim.x * blockDim.x) {
    uint4 k = make_uint4(kEmpty, kEmpty, kEmpty, kEmpty), t = make_uint4(0, 0, 0, 0);
    if (q < quads) {
      k = ld_cg_v4u(dv.keys + 4 * q);
      t = ld_cg_v4u(dv.ts + 4 * q);
    }
    const uint32_t kk[4] = {k.x, k.y, k.z, k.w}, tt[4] = {t.x, t.y, t.z, t.w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const bool live = kk[j] != kEmpty && tt[j] < epoch;
      const uint32_t a = live ? min(epoch - tt[j], (uint32_t)(kAgeBins - 1)) : 0xFFFFFFFFu;
      if (!dv.bytes) {  // equal rows: one shared-memory atomic per distinct age in the warp
        const unsigned grp = __match_any_sync(kFull, a);
        if (live && lane == __ffs(grp) - 1) atomicAdd(&h[a], (uint32_t)__popc(grp) * (uint32_t)(dv.dim >> 3));
      } else if (live) {
        atomicAdd(&h[a], way_units(dv, 4 * q + j));
      }
    }
  }
  __syncthreads();
  pdl_trigger();
  for (int i = threadIdx.x; i < kAgeBins; i += blockDim.x)
    if (h[i]) atomicAdd(ea.hist + i, 32ull * h[i]);
}

template <int = 0>
__global__ void __launch_bounds__(256) ke_evict_kernel(const __grid_constant__ Dev dv, const __grid_constant__ KEArgs ea) {
  __shared__ unsigned long long sh[kAgeBins];
  __shared__ unsigned long long part[256];
  __shared__ uint32_t sA;
  __shared__ int s_last;
  pdl_wait();
  const uint32_t epoch = *(volatile uint32_t*)&dv.ctl->epoch - 1u;
  const long long occ = *(volatile long long*)&dv.ctl->ke_occ;  // KE1's snapshot: the same in every CTA
  if (occ <= ea.hi) {  // every CTA takes this exit together (no histogram was built)
    pdl_trigger();
    return;
  }
  // threshold: the largest class A with S(A) = sum_{a >= A} bytes(a) >= occ - lo, else 1
  // (the oracle's loop "oldest class first while bytes > lo")
  const unsigned long long need = (unsigned long long)(occ - ea.lo);
  constexpr int kPer = kAgeBins / 256;
  unsigned long long mine = 0;
  for (int i = 0; i < kPer; ++i) {
    const int a = threadIdx.x * kPer + i;
    sh[a] = ld_cg_u64(ea.hist + a);
    mine += sh[a];
  }
  part[threadIdx.x] = mine;
  if (threadIdx.x == 0) sA = 1;
  __syncthreads();
  if (threadIdx.x == 0) {  // inclusive suffix sums of the 256 partials
    unsigned long long run = 0;
    for (int j = 255; j >= 0; --j) {
      run += part[j];
      part[j] = run;
    }
  }
  __syncthreads();
  unsigned long long S = threadIdx.x < 255 ? part[threadIdx.x + 1] : 0ull;
  if (S < need) {
    for (int a = threadIdx.x * kPer + kPer - 1; a >= threadIdx.x * kPer && a >= 1; --a) {
      S += sh[a];
      if (S >= need) {
        atomicMax(&sA, (uint32_t)a);
        break;
      }
    }
  }
  __syncthreads();
  const uint32_t A = sA;
  pdl_trigger();
  unsigned ev = 0;
  unsigned long long units = 0;
  const size_t ways = (size_t)dv.sets * 32u;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < ways; i += (size_t)gridDim.x * blockDim.x) {
    const uint32_t k = ld_cg_u32(dv.keys + i), t = ld_cg_u32(dv.ts + i);
    if (k == kEmpty || t >= epoch || min(epoch - t, (uint32_t)(kAgeBins - 1)) < A) continue;
    units += way_units(dv, i);
    dv.keys[i] = kEmpty;
    dv.ts[i] = 0;
    ++ev;
  }
  ev = __reduce_add_sync(kFull, ev);
#pragma unroll
  for (int o = 16; o; o >>= 1) units += __shfl_xor_sync(kFull, units, o);
  if ((threadIdx.x & 31) == 0 && ev) {
    atomicAdd(dv.stats + (blockIdx.x % kStripes) * kNumCtr + C_EVICTED, (unsigned long long)ev);
    atomicAdd((unsigned long long*)&dv.ctl->occ_bytes, (unsigned long long)(-(long long)(32ull * units)));
  }
  // the last CTA (every CTA has read the histogram by then) clears it for the next scan
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const uint32_t prev = atomicAdd(&dv.ctl->ke_done, 1u);
    s_last = prev == gridDim.x - 1;
    if (s_last) atomicAdd(dv.stats + C_SCANS, 1ull);
  }
  __syncthreads();
  if (s_last) {
    for (int i = threadIdx.x; i < kAgeBins; i += blockDim.x) ea.hist[i] = 0;
    if (threadIdx.x == 0) dv.ctl->ke_done = 0;
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
