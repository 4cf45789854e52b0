// kernels_f64_r9.cu -- dslash_kernel instantiations: links double, vectors double, long-link recon 9.
#include "kernels_inst.cuh"

HISQ_DEFINE_PICK(pick_f64_r9, double, double, 9)
