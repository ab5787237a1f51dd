// kern_f64_r5_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for double, r = 5.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f64_r5_ax, double, 5)
