// k_miss.cu — instantiates the miss kernel (KM): one specialisation per uniform row
// width (its register budget sized for that width alone) and one for the bytes layout
// (mixed widths, every class in turn), plus the static per-table mode with mixed widths.
#include "fns.h"

namespace fl {

KmFn km_fn(bool bytes, int dim) {
  if (bytes) return km_kernel<true, 0>;
  switch (dim) {
    case 8: return km_kernel<false, 8>;
    case 16: return km_kernel<false, 16>;
    case 32: return km_kernel<false, 32>;
    case 64: return km_kernel<false, 64>;
    case 128: return km_kernel<false, 128>;
    case 256: return km_kernel<false, 256>;
    default: return km_kernel<false, 0>;  // several widths in uniform per-table partitions (static mode)
  }
}

}  // namespace fl
