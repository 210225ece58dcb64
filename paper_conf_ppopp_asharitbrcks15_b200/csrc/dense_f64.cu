// dense_f64.cu -- fp64 instantiations of the dense kernels (dense_kernels.cuh).
#include "dense_kernels.cuh"

namespace fp {
DenseKFn dense_pick_f64(bool has_y, int variant, int chunk_bytes, int vs, int nch) {
  return has_y ? pick_t<double, true>(variant, chunk_bytes, vs, nch) : pick_t<double, false>(variant, chunk_bytes, vs, nch);
}
}  // namespace fp
