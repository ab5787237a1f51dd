// kern_f64_r1_dg.cu -- Div / Grad application stencils (divgrad.cuh) for double, r = 1.
#include "kern_inst.cuh"
STENCIL_REGISTER_DG(register_f64_r1_dg, double, 1)
