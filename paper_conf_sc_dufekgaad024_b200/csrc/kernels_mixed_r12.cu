// kernels_mixed_r12.cu -- dslash_kernel instantiations: links float, vectors double, long-link recon 12.
#include "kernels_inst.cuh"

HISQ_DEFINE_PICK(pick_mixed_r12, float, double, 12)
