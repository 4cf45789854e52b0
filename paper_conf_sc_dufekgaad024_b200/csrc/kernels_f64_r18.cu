// kernels_f64_r18.cu -- dslash_kernel instantiations: links double, vectors double, long-link recon 18.
#include "kernels_inst.cuh"

HISQ_DEFINE_PICK(pick_f64_r18, double, double, 18)
