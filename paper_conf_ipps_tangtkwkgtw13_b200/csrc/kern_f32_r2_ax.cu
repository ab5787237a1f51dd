// kern_f32_r2_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for float, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f32_r2_ax, float, 2)
