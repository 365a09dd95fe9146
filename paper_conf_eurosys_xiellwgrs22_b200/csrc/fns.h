// fns.h — host-side handles of the device kernels.
//
// The kernels are compiled in separate translation units (k_query.cu, k_miss.cu,
// k_misc.cu) so the build parallelises and every kernel gets its own register budget;
// the host code (fleche.cu) launches them through these function pointers (the host
// stubs, registered by the translation unit that instantiates each kernel).
#pragma once
#include <cstdint>

#include "kernels.cuh"
#include "shard.cuh"

namespace fl {

template <int MAXT> using KqFn = void (*)(QArgs<MAXT>, Dev);
template <int MAXT> using KpFn = void (*)(PArgs<MAXT>, const TableInfo*);
template <int MAXT> using KrFn = void (*)(RArgs<MAXT>, RouteDev, const TableInfo*);
template <int MAXT> using KrsFn = void (*)(RArgs<MAXT>, RouteDev, const float*, const uint8_t*, float*, PeerArgs);
using KmFn = void (*)(Dev, KMArgs);
using ProbeFn = void (*)(const float*, uint64_t, int64_t, uint64_t, float*);
using KpkFn = void (*)(RouteDev, uint32_t*, int64_t*, PeerKeys);
using KeFn = void (*)(Dev, KEArgs);

template <int MAXT> KqFn<MAXT> kq_fn(int tma_dim = 0);  // fused query; tma_dim 32/64: bulk-copy hit gather (k_query.cu)
template <int MAXT> KqFn<MAXT> kg_fn();   // decoupled hit copy (k_query.cu)
template <int MAXT> KpFn<MAXT> kp_fn();   // pooling (k_query.cu)
KmFn km_fn(bool bytes, int dim);          // miss kernel + restore (cooperative): bytes layout / uniform width dim / 0 = per class (k_miss.cu)
KeFn ke_hist_fn();                        // watermark scan: age histogram (k_misc.cu)
KeFn ke_evict_fn();                       // watermark scan: threshold + evict (k_misc.cu)
ProbeFn probe_fn(int dim);                // host-link probe (k_misc.cu)
template <int MAXT> KrFn<MAXT> kr_fn();   // key-sharded route (k_misc.cu)
KpkFn kpk_fn();                           // key-sharded pack (k_misc.cu)
template <int MAXT> KrsFn<MAXT> krs_fn(int dim);  // key-sharded restore (k_misc.cu)

}  // namespace fl
