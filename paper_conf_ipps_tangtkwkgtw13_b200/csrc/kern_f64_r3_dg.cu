// kern_f64_r3_dg.cu -- Div / Grad application stencils (divgrad.cuh) for double, r = 3.
#include "kern_inst.cuh"
STENCIL_REGISTER_DG(register_f64_r3_dg, double, 3)
