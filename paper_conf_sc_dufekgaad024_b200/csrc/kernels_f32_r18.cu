// kernels_f32_r18.cu -- dslash_kernel instantiations: links float, vectors float, long-link recon 18.
#include "kernels_inst.cuh"

HISQ_DEFINE_PICK(pick_f32_r18, float, float, 18)
