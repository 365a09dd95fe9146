// k_query.cu — instantiates the query-side kernels (KQ, KG, KP) for the table-count
// tiers the host dispatches to (n <= 32, <= 128, <= FLECHE_MAX_TABLES).
#include "fleche.h"
#include "fns.h"

namespace fl {

template <int MAXT> KqFn<MAXT> kq_fn(int tma_dim) {
  switch (tma_dim) {
    case 32: return kq_kernel<MAXT, 32>;
    case 64: return kq_kernel<MAXT, 64>;
    default: return kq_kernel<MAXT, 0>;
  }
}
template <int MAXT> KqFn<MAXT> kg_fn() { return kg_kernel<MAXT>; }
template <int MAXT> KpFn<MAXT> kp_fn() { return kp_kernel<MAXT>; }

#define FL_INST(M)                   \
  template KqFn<M> kq_fn<M>(int);    \
  template KqFn<M> kg_fn<M>();       \
  template KpFn<M> kp_fn<M>();
FL_INST(32)
FL_INST(128)
FL_INST(FLECHE_MAX_TABLES)
#undef FL_INST

}  // namespace fl
