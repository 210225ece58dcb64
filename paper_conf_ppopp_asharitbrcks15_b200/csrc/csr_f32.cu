// csr_f32.cu -- float instantiations of the CSR kernels (csr_kernels.cuh).
#include "csr_kernels.cuh"

namespace fp {
CsrKFn csr_pick_f32(int ym, int mode, int vs, int k) { return csr_pick_t<float>(ym, mode, vs, k); }
}  // namespace fp
