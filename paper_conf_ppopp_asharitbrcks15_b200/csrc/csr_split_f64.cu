// csr_split_f64.cu -- double instantiations of the column-split cluster kernel (csr_colsplit.cuh).
#include "csr_kernels.cuh"

namespace fp {
SplitKFn csr_pick_colsplit_f64(int ym, int cs, int nb) { return csr_pick_colsplit_t<double>(ym, cs, nb); }
}  // namespace fp
