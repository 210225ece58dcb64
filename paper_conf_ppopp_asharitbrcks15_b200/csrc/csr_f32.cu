// csr_f32.cu -- float dispatch of the CSR kernels (csr_kernels.cuh); the instantiations live in
// csr_f32_y{0,1,2}.cu, one translation unit per y mode so that they compile in parallel.
#include "csr_kernels.cuh"

namespace fp {
CsrKFn csr_pick_f32_y0(int mode, int vs, int k);
CsrKFn csr_pick_f32_y1(int mode, int vs, int k);
CsrKFn csr_pick_f32_y2(int mode, int vs, int k);
CsrKFn csr_pick_f32(int ym, int mode, int vs, int k) {
  switch (ym) {
    case 0: return csr_pick_f32_y0(mode, vs, k);
    case 1: return csr_pick_f32_y1(mode, vs, k);
    case 2: return csr_pick_f32_y2(mode, vs, k);
    default: return nullptr;
  }
}
}  // namespace fp
