// csr_f32_y2.cu -- float instantiations of the CSR kernels for y mode 2 (0 = no y, Table 1
// row 1; 1 = Eq. (1); 2 = Eq. (1) with a row epilogue).
#include "csr_kernels.cuh"

namespace fp {
CsrKFn csr_pick_f32_y2(int mode, int vs, int k) { return csr_pick_m<float, 2>(mode, vs, k); }
}  // namespace fp
