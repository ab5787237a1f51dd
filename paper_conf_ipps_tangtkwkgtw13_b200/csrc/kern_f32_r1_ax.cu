// kern_f32_r1_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for float, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f32_r1_ax, float, 1)
