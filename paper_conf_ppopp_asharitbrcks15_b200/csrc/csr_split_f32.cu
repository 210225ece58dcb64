// csr_split_f32.cu -- float instantiations of the column-split cluster kernel (csr_colsplit.cuh).
#include "csr_kernels.cuh"

namespace fp {
SplitKFn csr_pick_colsplit_f32(int ym, int cs, int nb) { return csr_pick_colsplit_t<float>(ym, cs, nb); }
}  // namespace fp
