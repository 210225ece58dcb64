// csr_f64.cu -- double instantiations of the CSR kernels (csr_kernels.cuh).
#include "csr_kernels.cuh"

namespace fp {
CsrKFn csr_pick_f64(int ym, int mode, int vs, int k) { return csr_pick_t<double>(ym, mode, vs, k); }
}  // namespace fp
