// kern_f32_r5_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for float, r = 5.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f32_r5_ax, float, 5)
