// kern_f64_r4_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for double, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f64_r4_ax, double, 4)
