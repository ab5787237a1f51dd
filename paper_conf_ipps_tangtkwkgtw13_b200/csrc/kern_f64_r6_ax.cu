// kern_f64_r6_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for double, r = 6.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f64_r6_ax, double, 6)
