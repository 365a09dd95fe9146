// k_misc.cu — instantiates the watermark scan kernels, the host-link probe and the
// key-sharded route / pack / restore kernels.
#include "fleche.h"
#include "fns.h"

namespace fl {

KeFn ke_hist_fn() { return ke_hist_kernel<0>; }
KeFn ke_evict_fn() { return ke_evict_kernel<0>; }

ProbeFn probe_fn(int dim) {
  switch (dim) {
    case 32: return probe_host_kernel<32>;
    case 64: return probe_host_kernel<64>;
    case 128: return probe_host_kernel<128>;
    case 256: return probe_host_kernel<256>;
    default: return nullptr;
  }
}

KpkFn kpk_fn() { return kpk_kernel<0>; }

template <int MAXT> KrFn<MAXT> kr_fn() { return kr_kernel<MAXT>; }

template <int MAXT> KrsFn<MAXT> krs_fn(int dim) {
  switch (dim) {
    case 8: return krs_kernel<MAXT, 8>;
    case 16: return krs_kernel<MAXT, 16>;
    case 32: return krs_kernel<MAXT, 32>;
    case 64: return krs_kernel<MAXT, 64>;
    case 128: return krs_kernel<MAXT, 128>;
    case 256: return krs_kernel<MAXT, 256>;
    default: return nullptr;
  }
}

#define FL_INST(M)                      \
  template KrFn<M> kr_fn<M>();          \
  template KrsFn<M> krs_fn<M>(int);
FL_INST(32)
FL_INST(128)
FL_INST(FLECHE_MAX_TABLES)
#undef FL_INST

}  // namespace fl
