// kernels_mixed_r9.cu -- dslash_kernel instantiations: links float, vectors double, long-link recon 9.
#include "kernels_inst.cuh"

HISQ_DEFINE_PICK(pick_mixed_r9, float, double, 9)
