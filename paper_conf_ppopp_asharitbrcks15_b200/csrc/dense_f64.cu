// dense_f64.cu -- double instantiations of the dense kernels (dense_kernels.cuh).
#include "dense_kernels.cuh"

namespace fp {
// ym: 0 = no y (Table 1 row 1), 1 = Eq. (1), 2 = Eq. (1) with a row epilogue
DenseKFn dense_pick_f64(int ym, int variant, int chunk_bytes, int vs, int nch, int tma) {
  switch (ym) {
    case 0: return pick_t<double, 0>(variant, chunk_bytes, vs, nch, tma);
    case 1: return pick_t<double, 1>(variant, chunk_bytes, vs, nch, tma);
    case 2: return pick_t<double, 2>(variant, chunk_bytes, vs, nch, tma);
    default: return nullptr;
  }
}
}  // namespace fp
