// csr_f64.cu -- double instantiations of the CSR kernels (csr_kernels.cuh).
#include "csr_kernels.cuh"

namespace fp {
CsrKFn csr_pick_f64(bool has_y, int mode, int vs, int k) { return csr_pick_t<double>(has_y, mode, vs, k); }
}  // namespace fp
