/*
 * include/fleche.h — C ABI of libfleche.so, the B200 (sm_100a) flat embedding cache.
 *
 * What it computes (paper: /root/reference/PAPER.md, cited P:L<a>-<b>):
 *   A DLRM has embedding tables E_0..E_{n-1}; E_t has capacity (corpus size) c_t and
 *   value dimension d_t.  A query for table t carries an ID list
 *   ID_List_t and fills the output matrix O_t of shape len(ID_List_t) x d_t with the
 *   rows E_t[id].  Fleche answers the queries of ALL tables through one
 *   flat GPU-resident cache shared by every table (flat cache, P:L503-507,
 *   P:L513-528) with one fused, self-identified launch and
 *   "still supports the original interface of multi-cache queries":
 *   that interface is fleche_query below.  Rows that miss in HBM are read straight
 *   from the CPU-DRAM layer by the GPU (unified index); missed rows are
 *   inserted with approximate-LRU replacement.
 *
 * The result (`out`) is the plain definition: out row = E_t[id], bit for bit; the
 * cache only changes how fast it is produced.
 *
 * Threading / ordering: a ctx is not thread-safe.  Calls on one ctx execute on the
 * device in call order, even when they are issued on different streams (the
 * library chains them with an internal event).  Every call except fleche_stats,
 * fleche_debug_snapshot and fleche_destroy is asynchronous with respect to the host.
 *
 * Errors: status codes only; nothing is thrown across the ABI.  Host-side argument
 * validation returns FLECHE_EINVAL with nothing enqueued.  A CUDA error poisons the
 * ctx: that call returns FLECHE_ECUDA and every later call FLECHE_ESTATE.
 */
#ifndef FLECHE_H_
#define FLECHE_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct fleche_ctx fleche_ctx; /* opaque; one per (process, GPU) */
typedef void* fleche_stream;           /* a cudaStream_t; NULL = legacy default stream */

typedef enum {
  FLECHE_OK = 0,
  FLECHE_EINVAL = -1, /* bad argument; nothing was enqueued                                    */
  FLECHE_ENOMEM = -2, /* device or pinned-host allocation failed                               */
  FLECHE_ECUDA = -3,  /* a CUDA call failed; the ctx is now poisoned                          */
  FLECHE_ENCCL = -4,  /* reserved for the key-sharded multi-GPU mode                          */
  FLECHE_ERANGE = -5, /* fleche_stats: some query since the last reset carried an ID outside
                         [0, c_t); the stats are still valid (see fleche_query)               */
  FLECHE_ESTATE = -6  /* ctx poisoned by an earlier CUDA error                                */
} fleche_status;

#define FLECHE_MAX_TABLES 512 /* per-call table arguments travel as kernel parameters (<= 32 KB) */

typedef struct {
  int32_t num_tables;            /* n, 1 <= n <= FLECHE_MAX_TABLES                               */
  const int64_t* cardinalities;  /* [n] host array: c_t >= 1 rows of table t                    */
  const int32_t* dims;           /* [n] host array: d_t in {8, 16, 32, 64, 128, 256} (rows are moved
                                    as 16-byte vectors by warp-shaped kernels specialised per
                                    width).  One width for all tables -> uniform layout (32-way
                                    sets of equal rows); mixed widths -> bytes layout (32-way sets
                                    sharing a 4 KiB row region each: one byte budget for every
                                    width, the flat cache's elastic per-table capacity, P:L801-804;
                                    slabs per width as in Fig 5c).                    */
  uint64_t cache_bytes;          /* HBM budget for cached embedding ROWS (the paper expresses the
                                    cache size as a fraction of all table bytes);
                                    uniform: capacity = floor(cache_bytes / (4 d)) rows; bytes:
                                    floor(cache_bytes / 4096) sets x 4096 B.  The index and the
                                    scratch are reported separately in index_bytes.               */
  const float* const* host_tables;/* [n] host array of host pointers: E_t row-major c_t x d_t fp32,
                                    16-byte aligned, caller-owned, must outlive the ctx.  The ctx
                                    page-locks and maps them (cudaHostRegister Mapped|Portable)
                                    unless they are already registered/pinned; the GPU then reads
                                    missed rows with zero-copy loads over the host link.          */
  int64_t max_lookups;           /* upper bound on sum_t lengths[t] per fleche_query call; sizes
                                    every per-batch scratch buffer once at create (no allocation
                                    on the query path)                                */
  int32_t device;                /* CUDA device ordinal                                           */
  double admit_prob;             /* admission probability p; <= 0 or >= 1 => admit
                                    every miss.  Coin: splitmix64(admit_seed ^ fk ^ (batch << 32))
                                    < p * 2^64, batch = 0-based query count (R8)        */
  uint64_t admit_seed;
  uint32_t hash_seed;            /* set index = (fmix32(fk ^ hash_seed) * S) >> 32 (R12)  */
  uint32_t flags;                /* bitwise OR of FLECHE_FLAG_*; other bits must be 0              */
  int32_t key_bits;              /* flat-key width B.  0 (or >= B_min) = the exact size-aware code
                                    (P:L640-652).  1 <= B < B_min = short flat keys (P:L646-649,
                                    DESIGN.md reading R24): the smallest tables keep exact codes, the
                                    others share the space left in proportion to their sizes with
                                    their feature IDs hashed into g_t bits, so out row =
                                    E_t[h_t(id)] (the model's table is indexed by the hashed
                                    feature; IDs that collide share one row and one cache entry).
                                    fleche_get_encoding reports g_t.  Not with the key-sharded mode. */
  int32_t reserved;              /* must be 0                                                      */
} fleche_config;

/* Flag bit 0x1 is reserved (was an L2-prefetch experiment, measured slower and removed;
 * profiles/README.md, round 1): fleche_create rejects it with FLECHE_EINVAL. */
/* Baseline / ablation modes (the paper's comparison point):
 * STATIC_PER_TABLE: replace the flat cache by one static cache per table, each with
 *   floor(frac * c_t) rows where frac = cache_bytes / sum_t 4 c_t d_t ("the same
 *   proportion of cache size for all embedding tables"; reading R17), each a
 *   32-way set-associative partition of its own (uniform layout per table);
 * PER_TABLE_LAUNCH: launch the query kernel once per table (n launches instead of one
 *   self-identified launch; the kernel-maintenance cost of P:L479-497). */
#define FLECHE_FLAG_STATIC_PER_TABLE 0x2u
#define FLECHE_FLAG_PER_TABLE_LAUNCH 0x4u
/* HOST_ASSIST: host-assisted miss fetch -- the paper's decoupled workflow with the
 * CPU-DRAM layer queried "ahead", as soon as the indexing kernel knows which keys miss,
 * in parallel with the GPU's hit copy (Fig 8b; CPU-DRAM layer P:L177-178).
 * The unified index (Fig 8c) lets the GPU read each missed row where it
 * lies in the host tables.  On this platform scattered zero-copy reads are capped by
 * address translation (~80 M rows/s beyond a ~1 GiB span), while host cores
 * gather scattered rows at ~60 GB/s, so by DEFAULT a ctx whose host tier spans >= 1 GiB
 * (>= 8 host CPUs; not the static per-table or per-table-launch ablations) runs host
 * threads that gather a share of the batch's
 * unique missed rows into a contiguous pinned staging buffer, which the miss kernel reads
 * over the link at its full rate while it reads the rest zero-copy itself (two paths at
 * once).  HOST_ASSIST forces it on (also for small tiers),
 * NO_HOST_ASSIST off.  Requests travel GPU -> host through pinned memory, tagged with the
 * batch epoch: the query kernel's owner lanes write them to HBM and a few side CTAs of the
 * same launch forward them to the host list 1 KiB per staging block (FLECHE_HA_FWD = CTAs,
 * default 8; 0 = the lanes write the host list directly); the query kernel's first CTA
 * writes a start word (the threads stream the requests as they come) and its last CTA
 * rings the doorbell with the counts; ONE miss-kernel warp polls the threads' progress
 * words and mirrors them into HBM for the others (no host sync, no extra launch: the path
 * stays asynchronous and graph-capturable).  From FLECHE_HA_EARLY_MIN lookups per batch
 * (default 524288) 16 more side CTAs copy already staged blocks into HBM while the
 * lookups run (FLECHE_HA_EARLY=0 turns that off).  Blocks not staged
 * within FLECHE_HA_TIMEOUT_US (default 2000) are read zero-copy from the tables, so
 * correctness never depends on the threads.  Env: FLECHE_HA_THREADS (default
 * min(12, CPUs - 4)), FLECHE_HA_STAGE_KB (staging per epoch parity, default 131072, or
 * 524288 with several row widths, shared equally by the widths; a width's misses beyond its
 * rows are read zero-copy), FLECHE_HA_FRAC (fixes the share of the staging blocks the host
 * threads take; default: tuned online, see fleche_stats.ui_share_ppm), FLECHE_HA_MIN_ROWS
 * (batches with fewer unique misses stay all zero-copy, default 1024).  Not with
 * PER_TABLE_LAUNCH (FLECHE_EINVAL).  `out`, hits and every cache decision are identical
 * with and without it; only where the missed rows are read from changes. */
#define FLECHE_FLAG_HOST_ASSIST 0x8u
#define FLECHE_FLAG_NO_HOST_ASSIST 0x20u
/* FUSED_HIT_COPY: the query kernel copies each hit row itself (probe and copy in one
 * kernel, the fused design; the default since round 2, measured faster with the
 * host-assisted miss fetch) even when FLECHE_DECOUPLE_MIN (lookups per batch, env) asks for
 * the decoupled copy (Fig 8b), where the query kernel only indexes and a copy
 * kernel on a side stream moves the hit rows while the miss kernel fetches the misses.
 * The paper's decoupling on/off comparison (Exp #7).  `out` and every
 * counter are identical either way. */
#define FLECHE_FLAG_FUSED_HIT_COPY 0x10u

typedef struct {
  uint64_t batches;            /* query calls                                                       */
  uint64_t lookups;            /* IDs looked up (valid + invalid)                                   */
  uint64_t hits;               /* lookups whose key was cached before the batch started             */
  uint64_t misses;             /* valid lookups that were not cached (duplicates included)          */
  uint64_t invalid;            /* IDs outside [0, c_t): zero row, never cached                      */
  uint64_t unique_keys;        /* unique valid keys per batch, summed                               */
  uint64_t unique_hits;
  uint64_t unique_misses;      /* = rows read from the host tier                                    */
  uint64_t inserted;           /* rows admitted into the cache                                      */
  uint64_t evicted;            /* cached rows replaced                                              */
  uint64_t bypassed;           /* unique misses not inserted (admission coin, or every way of the
                                  set was read/written in the same batch)                          */
  uint64_t occupancy_bytes;    /* rows currently cached x row bytes (<= capacity_bytes)             */
  uint64_t capacity_bytes;     /* capacity rows x row bytes                                         */
  uint64_t index_bytes;        /* HBM used by index + scratch (not counted in cache_bytes)          */
  uint64_t host_bytes_fetched; /* bytes read from the host tier over the host link                  */
  uint64_t kernels_launched;   /* kernels this ctx launched                                         */
  uint64_t assisted_rows;      /* HOST_ASSIST: unique misses read from the host threads' staging    */
  uint64_t assist_timeouts;    /* HOST_ASSIST: staging blocks fetched zero-copy after the timeout   */
  uint64_t scans;              /* fleche_set_watermarks: batches whose full-table scan evicted      */
  uint64_t ui_share_ppm;       /* host-assisted ctx: the unified index's current share of a batch's
                                  staging blocks (GPU zero-copy reads; the host threads take the
                                  rest), in parts per million, as tuned by the loop of P:L861-872;
                                  0 without host assistance                                         */
} fleche_stats_t;

/* Create a cache for the tables in *cfg on cfg->device.  Allocates every device
 * buffer once.  Returns FLECHE_EINVAL for an invalid configuration,
 * including tables whose size-aware flat keys do not fit in 32 bits. */
fleche_status fleche_create(const fleche_config* cfg, fleche_ctx** out);

/* One batch of one-hot lookups for every table.
 *   ids[t]     : DEVICE pointer to lengths[t] int64 IDs of table t (may be NULL if
 *                lengths[t] == 0); ids itself is a HOST array of n pointers.
 *   lengths[t] : HOST array, len(ID_List_t) >= 0; sum <= max_lookups.
 *   out        : DEVICE fp32 buffer, table-major concatenation of O_t: table t starts
 *                at float offset sum_{u<t} lengths[u] * d_u; row j of O_t = E_t[ids[t][j]].
 *                16-byte aligned.
 *   stream     : cudaStream_t the work is enqueued on.
 * IDs outside [0, c_t) (reading R15) yield a zero row, count as `invalid`, are never
 * cached, and make the next fleche_stats return FLECHE_ERANGE.  Caller owns ids and
 * out; they must stay valid until the stream has passed this call.  Enqueues 2
 * kernels on `stream` -- the query kernel (KQ: probe, hit gather, miss dedup) and the
 * miss kernel (KM, a cooperative launch: miss fetch, insert, restore of duplicate misses) -- plus,
 * only when decoupling is enabled (FLECHE_DECOUPLE_MIN lookups per batch; off by default),
 * the decoupled hit copy (KG) on a ctx-owned side stream that `stream` joins; with watermarks set (fleche_set_watermarks)
 * 2 scan kernels follow.  Never blocks the host. */
fleche_status fleche_query(fleche_ctx* ctx, const int64_t* const* ids, const int64_t* lengths, float* out,
                           fleche_stream stream);

/* Warm start (the paper warms the cache by first issuing requests): one
 * batch of one-hot lookups exactly as fleche_query (same policy, same counters: it is a
 * batch of the cache), whose rows go to a ctx-owned scratch buffer (allocated at the
 * first call, grown when a larger batch comes) instead of a caller buffer.  ids / lengths
 * as in fleche_query.  Asynchronous. */
fleche_status fleche_prefill(fleche_ctx* ctx, const int64_t* const* ids, const int64_t* lengths, fleche_stream stream);

/* One batch of multi-hot lookups with sum pooling per bag (pooling).
 *   ids[t]     : DEVICE pointer to nnz[t] int64 IDs of table t (all bags, concatenated).
 *   offsets[t] : DEVICE pointer to bags[t] + 1 int64 CSR offsets into ids[t]:
 *                bag b = ids[t][offsets[t][b] .. offsets[t][b+1]); offsets[t][0] = 0 and
 *                offsets[t][bags[t]] = nnz[t] (the caller guarantees this; not checked).
 *   bags, nnz  : HOST arrays; sum_t nnz[t] <= max_lookups.
 *   out        : DEVICE fp32, table t starts at float offset sum_{u<t} bags[u] * d_u; bag b's
 *                row = fp32 sum of E_t[id] over its valid IDs, accumulated sequentially in
 *                bag order (reading R16: the oracle's order, so results are bit-identical);
 *                an empty bag gives a zero row; invalid IDs contribute nothing.
 * Every ID is a lookup for the cache (hit/miss/insert as in fleche_query).  Enqueues
 * 3 kernels (query, miss + restore, pooling); the per-ID rows are staged in a ctx-owned buffer
 * (max_lookups x max d floats, allocated at the first pooled call). */
fleche_status fleche_query_pooled(fleche_ctx* ctx, const int64_t* const* ids, const int64_t* const* offsets,
                                  const int64_t* bags, const int64_t* nnz, float* out, fleche_stream stream);

/* Same lookups with HOST buffers: ids[t] are host pointers (ideally pinned), out is a
 * host buffer.  Enqueues host->device copies of the IDs and the query on a ctx-owned
 * stream (after the ctx's previous batch, NOT after `stream`: the host IDs must be final
 * when the call is made and stay unchanged until `stream` is synchronised), and the
 * device->host copy of out on a second ctx-owned stream (after the query and after
 * whatever `stream` holds) from one of two staging buffers, so call k's output copy
 * overlaps call k+1's lookups; `stream` waits for the copy.  (Env FLECHE_HOST_ORDERED=1
 * also orders the lookups after `stream`, serialising copy k and lookups k+1.)
 * Asynchronous: out is complete once `stream` is synchronised (ctx-owned device staging,
 * allocated at the first call). */
fleche_status fleche_query_host(fleche_ctx* ctx, const int64_t* const* ids, const int64_t* lengths, float* out,
                                fleche_stream stream);

/* Counters accumulated since create / the last reset.  Blocks until the ctx's
 * work has finished.  Returns FLECHE_ERANGE (with *out filled) if an invalid ID
 * was seen since the last reset. */
fleche_status fleche_stats(fleche_ctx* ctx, fleche_stats_t* out);
fleche_status fleche_reset_stats(fleche_ctx* ctx);

/* Watermark (full-scan) eviction, the paper's eviction trigger ("when the
 * utilization of the memory pool exceeds a certain threshold, FC performs cache eviction
 * with a full table scan and keeps evicting cold embeddings until memory utilization
 * falls below another threshold"; no values are given).  Reading R23: after
 * every later batch, if the cached row bytes exceed floor(hi * capacity_bytes), the ctx
 * scans the whole index and evicts, oldest first, whole age classes (age = batches since
 * the entry was last read or written, saturated at 4095) of the entries NOT touched in
 * that batch (epoch-based reclamation), until the bytes are <=
 * floor(lo * capacity_bytes) or no untouched entry is left.  On-demand eviction inside
 * a full set stays as in the canonical policy.  hi >= 1 turns the scan off (default).
 * Adds 2 kernel launches per batch (both exit at once below hi).  Blocks until the
 * ctx's queued work is done.  FLECHE_EINVAL: hi or lo <= 0, lo > hi, or a
 * FLECHE_FLAG_STATIC_PER_TABLE ctx. */
fleche_status fleche_set_watermarks(fleche_ctx* ctx, double hi, double lo);

/* Release every device buffer and host registration the ctx made. */
fleche_status fleche_destroy(fleche_ctx* ctx);

const char* fleche_strerror(fleche_status status);

/* Introspection for tests.
 * fleche_get_encoding: base[t] (first flat key of table t), fbits[t] (feature bits),
 *   *key_bits = minimal key width B_min of the size-aware code.
 * fleche_get_geometry: number of index sets S; uniform layout: capacity rows and row
 *   floats d; bytes layout: rows = 0 and row_floats = -(floats of one set's region).
 * fleche_debug_snapshot: blocking copy of the index (keys[S*32], ts[S*32]; uint32,
 *   EMPTY key = 0xFFFFFFFF) and of the slab (uniform: S*32 rows x d floats, row of way w
 *   of set s at (s*32 + w) * d; bytes: S regions) into host buffers of at least the
 *   given element counts.
 * fleche_debug_locations: bytes layout only: loc[S*32] = (size << 8) | offset of each
 *   way's row inside its set's region, both in 32-byte units. */
fleche_status fleche_get_encoding(fleche_ctx* ctx, uint64_t* base, int32_t* fbits, int32_t* key_bits);

/* The flat-key code fleche_create would build for these cardinalities, without a ctx or a
 * GPU (host-only; P:L640-652 size-aware coding, readings R3 and R24).
 *   cards[n] (host, c_t >= 1); key_bits = the config's key_bits (0 = exact code);
 *   out: base[n] (first flat key of table t), fbits[n] (feature bits f_t, or g_t for a
 *   hashed table), hashed[n] (1 = the table's feature IDs are hashed; may be NULL),
 *   *key_bits_out = the code's key width (B_min for the exact code).
 * Errors: FLECHE_EINVAL on null pointers, n outside [1, FLECHE_MAX_TABLES], c_t < 1,
 *   key_bits outside [0, 32], or a code that does not fit (exact code wider than 32 bits
 *   with key_bits = 0).  Caller owns every buffer. */
fleche_status fleche_encode(int32_t n, const int64_t* cards, int32_t key_bits, uint64_t* base, int32_t* fbits,
                            int32_t* hashed, int32_t* key_bits_out);
fleche_status fleche_get_geometry(fleche_ctx* ctx, int64_t* sets, int64_t* rows, int32_t* row_floats);
fleche_status fleche_debug_snapshot(fleche_ctx* ctx, uint32_t* keys, uint32_t* ts, size_t ways_cap, float* slab,
                                    size_t slab_floats_cap);
fleche_status fleche_debug_locations(fleche_ctx* ctx, uint16_t* loc, size_t ways_cap);

/* Key-sharded multi-GPU mode (the paper leaves multi-GPU caching to
 * future work).  Rank r of G caches only the keys it OWNS:
 * owner(fk) = (fmix32(fk ^ owner_seed ^ 0x85EBCA77) * G) >> 32, so the G per-GPU
 * budgets aggregate.  One batch on every rank (all calls on the same stream):
 *   1. fleche_route(ids, lengths, G, seed, send_keys, send_counts): dedups the batch's
 *      valid flat keys and writes them grouped by owner (send_keys[sum counts], uint32
 *      flat keys, DEVICE) with per-owner counts (send_counts[G], int64, DEVICE).
 *   2. the caller exchanges counts and keys with an all-to-all (NCCL over NVLink);
 *   3. fleche_query_keys(recv_keys, R, rows, flags): the owner answers R flat keys
 *      (its share of every rank's batch) with the ordinary query and miss kernels:
 *      rows[R x d] fp32 (DEVICE, row g answers key g), hit_flags[R] (DEVICE, 1 = hit;
 *      may be NULL); this is one batch (epoch) of the owner's cache;
 *   4. the caller returns rows (and flags) with an all-to-all, owners in rank order,
 *      each owner's rows in the order the keys were sent;
 *   5. fleche_restore(rows_back, flags_back, out): out (layout of fleche_query for the
 *      lengths of step 1) gets every lookup's row; invalid IDs give a zero row.
 * Uniform row widths only (FLECHE_EINVAL otherwise); G <= 64.
 * fleche_shard_stats: requester-side counters: lookups routed, lookups whose key hit
 * at its owner, invalid IDs, unique keys routed (summed over batches). */
fleche_status fleche_route(fleche_ctx* ctx, const int64_t* const* ids, const int64_t* lengths, int32_t world,
                           uint32_t owner_seed, uint32_t* send_keys, int64_t* send_counts, fleche_stream stream);
fleche_status fleche_query_keys(fleche_ctx* ctx, const uint32_t* keys, int64_t count, float* rows,
                                uint8_t* hit_flags, fleche_stream stream);
fleche_status fleche_restore(fleche_ctx* ctx, const float* rows, const uint8_t* hit_flags, float* out,
                             fleche_stream stream);
fleche_status fleche_shard_stats(fleche_ctx* ctx, uint64_t* lookups, uint64_t* hits, uint64_t* invalid,
                                 uint64_t* unique_routed);

/* Fused exchange for step 4-5 of the key-sharded batch (SURVEY §8(e) "fused variant"):
 * instead of returning rows with an all-to-all and restoring from the local copy, the
 * restore kernel reads every owner's answer in place over peer memory (NVLink P2P
 * loads through CUDA IPC mappings), so the row transfer is the restore's own loads.
 *   peer_rows[o]  : DEVICE pointer (valid in this process: own buffer for o == rank, an
 *                   fleche_ipc_open mapping otherwise) to owner o's `rows` of its
 *                   fleche_query_keys call of this batch;
 *   peer_flags[o] : same for its hit_flags (peer_flags itself may be NULL: no hit counts);
 *   peer_off[o]   : HOST int64: index of this rank's first key in owner o's received
 *                   order (= sum of the counts owner o received from ranks < this rank).
 * world must equal the last fleche_route's.  The caller orders the owners' queries before
 * this call on every rank (a stream-ordered barrier, e.g. an NCCL all-reduce of one
 * element) and keeps the owners' buffers unchanged until every rank has restored (double
 * buffering by batch parity).  out as in fleche_restore. */
fleche_status fleche_restore_p2p(fleche_ctx* ctx, int32_t world, const float* const* peer_rows,
                                 const uint8_t* const* peer_flags, const int64_t* peer_off, float* out,
                                 fleche_stream stream);
/* Fused exchange, key side: fleche_route whose pack step stores each unique key straight
 * into its owner's receive buffer (peer HBM through CUDA IPC) instead of send_keys:
 * peer_slots[o] = DEVICE pointer to this rank's slot in owner o's buffer (room for
 * max_lookups keys).  send_counts as in fleche_route.  The owner answers the keys of all
 * sources with fleche_query_keys_seg once every rank's route has completed (e.g. after
 * the counts all-gather, itself stream-ordered behind the routes). */
fleche_status fleche_route_p2p(fleche_ctx* ctx, const int64_t* const* ids, const int64_t* lengths, int32_t world,
                               uint32_t owner_seed, uint32_t* const* peer_slots, int64_t* send_counts,
                               fleche_stream stream);
/* fleche_query_keys over nseg segments (one per source rank, in rank order): segs[i] is a
 * DEVICE pointer to counts[i] (HOST) flat keys; row g of `rows` answers the g-th key of
 * their concatenation.  One batch of the owner's cache. */
fleche_status fleche_query_keys_seg(fleche_ctx* ctx, const uint32_t* const* segs, const int64_t* counts, int32_t nseg,
                                    float* rows, uint8_t* hit_flags, fleche_stream stream);
/* Sync-free fused exchange (no host read of any count per batch): the G x G matrix
 * counts_dev[src * G + owner] (int64, DEVICE, row-major) holds every rank's send_counts of
 * this batch, e.g. the stream-ordered all-gather of them (NCCL), and me = this rank.
 * fleche_query_keys_seg_dev answers segment src (counts_dev[src * G + me] keys at segs[src])
 * with a grid sized for the ctx's max_lookups that strides over the device-side total;
 * fleche_restore_p2p_dev computes this rank's offset in every owner's order on the device
 * (the sum of counts_dev[src * G + o] over src < me).  Otherwise as fleche_query_keys_seg /
 * fleche_restore_p2p; the owner's fleche_stats lookup count is not advanced (use
 * fleche_shard_stats).  FLECHE_EINVAL for bad pointers, world or me. */
fleche_status fleche_query_keys_seg_dev(fleche_ctx* ctx, const uint32_t* const* segs, const int64_t* counts_dev,
                                        int32_t world, int32_t me, float* rows, uint8_t* hit_flags,
                                        fleche_stream stream);
fleche_status fleche_restore_p2p_dev(fleche_ctx* ctx, int32_t world, const float* const* peer_rows,
                                     const uint8_t* const* peer_flags, const int64_t* counts_dev, int32_t me,
                                     float* out, fleche_stream stream);
/* CUDA IPC helpers for the fused exchange: export a device allocation (the base pointer
 * of a cudaMalloc allocation) as a 64-byte handle, map a peer process's handle into this
 * process (peer access enabled lazily), unmap it.  FLECHE_ECUDA on failure. */
fleche_status fleche_ipc_alloc(size_t bytes, void** dptr); /* a cudaMalloc allocation to export */
fleche_status fleche_ipc_free(void* dptr);
fleche_status fleche_ipc_handle(const void* dptr, uint8_t handle[64]);
fleche_status fleche_ipc_open(const uint8_t handle[64], void** dptr);
fleche_status fleche_ipc_close(void* dptr);

/* Diagnostics for measurement (bench.py).
 * fleche_set_profiling: when enabled, every later query records CUDA events on its
 *   stream around each of its kernels (adds ~3 event records per call).
 * fleche_kernel_times: blocking; summed device time (ms) of the query kernel (KQ) and
 *   of everything after it (*ki_ms: the miss kernel KM, which also restores duplicate
 *   misses, and the pooling kernel) over the profiled queries since the last call, and
 *   their count; resets the accumulation.
 * fleche_probe_host_read: measures random-row zero-copy read bandwidth of the host
 *   link: a kernel with the KQ miss-fetch access pattern reads `rows` rows of
 *   `row_bytes` (multiple of 16, <= 4096) at seeded random row indices of the mapped
 *   host buffer [host, host + bytes) (already registered, e.g. a ctx's table), timed
 *   with CUDA events on `stream`; *gbps = rows * row_bytes / time.  Blocking. */
fleche_status fleche_set_profiling(fleche_ctx* ctx, int enable);
fleche_status fleche_kernel_times(fleche_ctx* ctx, double* kq_ms, double* ki_ms, uint64_t* queries);
/* Same accumulation split per kernel: ms4 = {query (KQ), miss + restore (KM), 0 (the
 * former separate restore kernel, now inside KM), pooling (KP; 0 for one-hot)} summed
 * over the profiled queries; resets. */
fleche_status fleche_kernel_times_ex(fleche_ctx* ctx, double* ms4, uint64_t* queries);
/* Tools only: copy the device control block (sizeof = bytes >= its size) to host on a
 * private non-blocking stream, so it can be read while the ctx's streams are stuck. */
fleche_status fleche_debug_ctl(fleche_ctx* ctx, void* host, size_t bytes);
fleche_status fleche_probe_host_read(const void* host, uint64_t bytes, int32_t row_bytes, int64_t rows, uint64_t seed,
                                     fleche_stream stream, double* gbps);

#ifdef __cplusplus
}
#endif
#endif /* FLECHE_H_ */
