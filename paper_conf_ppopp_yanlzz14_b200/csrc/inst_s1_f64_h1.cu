// Precompiled strategy-1 (intermediate sums in registers) SpMV kernel instances: dtype double, block
// height 1, block widths {1,2,4,8} x thread tiles {4,8,16,32} x column modes (Table 1,
// P:305-319), restricted to T*h*w*sizeof(value) <= 512 bytes of values per thread.
#include "spmv_kernel.cuh"

namespace yaspmv {
void register_s1_f64_h1(std::vector<KernelEntry>& R) { reg_h<double, 1>(R); }
}  // namespace yaspmv
