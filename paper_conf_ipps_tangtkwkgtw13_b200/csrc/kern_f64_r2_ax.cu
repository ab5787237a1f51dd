// kern_f64_r2_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for double, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f64_r2_ax, double, 2)
