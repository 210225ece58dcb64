// dense_f32.cu -- fp32 instantiations of the dense kernels (dense_kernels.cuh).
#include "dense_kernels.cuh"

namespace fp {
DenseKFn dense_pick_f32(bool has_y, int variant, int chunk_bytes, int vs, int nch) {
  return has_y ? pick_t<float, true>(variant, chunk_bytes, vs, nch) : pick_t<float, false>(variant, chunk_bytes, vs, nch);
}
}  // namespace fp
