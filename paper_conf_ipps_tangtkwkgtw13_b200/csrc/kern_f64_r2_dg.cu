// kern_f64_r2_dg.cu -- Div / Grad application stencils (divgrad.cuh) for double, r = 2.
#include "kern_inst.cuh"
STENCIL_REGISTER_DG(register_f64_r2_dg, double, 2)
