// kernels_f32_r9.cu -- dslash_kernel instantiations: links float, vectors float, long-link recon 9.
#include "kernels_inst.cuh"

HISQ_DEFINE_PICK(pick_f32_r9, float, float, 9)
