// csr_f64_y1.cu -- double instantiations of the CSR kernels for y mode 1 (0 = no y, Table 1
// row 1; 1 = Eq. (1); 2 = Eq. (1) with a row epilogue).
#include "csr_kernels.cuh"

namespace fp {
CsrKFn csr_pick_f64_y1(int mode, int vs, int k) { return csr_pick_m<double, 1>(mode, vs, k); }
}  // namespace fp
