// kern_f32_r6_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for float, r = 6.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f32_r6_ax, float, 6)
