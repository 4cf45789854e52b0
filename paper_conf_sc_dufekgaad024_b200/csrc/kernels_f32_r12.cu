// kernels_f32_r12.cu -- dslash_kernel instantiations: links float, vectors float, long-link recon 12.
#include "kernels_inst.cuh"

HISQ_DEFINE_PICK(pick_f32_r12, float, float, 12)
