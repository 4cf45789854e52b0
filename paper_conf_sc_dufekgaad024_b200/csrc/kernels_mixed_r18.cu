// kernels_mixed_r18.cu -- dslash_kernel instantiations: links float, vectors double, long-link recon 18.
#include "kernels_inst.cuh"

HISQ_DEFINE_PICK(pick_mixed_r18, float, double, 18)
