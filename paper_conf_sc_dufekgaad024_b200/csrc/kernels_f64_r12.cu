// kernels_f64_r12.cu -- dslash_kernel instantiations: links double, vectors double, long-link recon 12.
#include "kernels_inst.cuh"

HISQ_DEFINE_PICK(pick_f64_r12, double, double, 12)
