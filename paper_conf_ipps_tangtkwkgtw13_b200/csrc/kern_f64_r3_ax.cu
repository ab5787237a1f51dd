// kern_f64_r3_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for double, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f64_r3_ax, double, 3)
