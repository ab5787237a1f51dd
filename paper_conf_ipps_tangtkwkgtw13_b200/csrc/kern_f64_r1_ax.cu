// kern_f64_r1_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for double, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f64_r1_ax, double, 1)
