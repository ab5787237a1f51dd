// kern_f32_r4_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for float, r = 4.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f32_r4_ax, float, 4)
