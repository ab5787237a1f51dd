// kern_f32_r3_ax.cu -- per-axis-coefficient sweep kernels (reading R3b) for float, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER_AX(register_f32_r3_ax, float, 3)
