// dispatch.h -- kernel selection across the per-precision translation units (kernels_*.cu).
#pragma once

#include "common.cuh"
#include "stencil.cuh"

namespace hisq {

typedef void (*StencilFn)(StencilParams);

// Each returns the dslash_kernel instantiation for (ghost, lanes 1/2/4, min blocks 2/3/4,
// right-hand sides per launch 1/2/4/8) of one (precision, long-link recon) pair.
StencilFn pick_f64_r18(bool ghost, int lanes, int minb, int nrhs);
StencilFn pick_f64_r12(bool ghost, int lanes, int minb, int nrhs);
StencilFn pick_f32_r18(bool ghost, int lanes, int minb, int nrhs);
StencilFn pick_f32_r12(bool ghost, int lanes, int minb, int nrhs);
StencilFn pick_mixed_r18(bool ghost, int lanes, int minb, int nrhs);
StencilFn pick_mixed_r12(bool ghost, int lanes, int minb, int nrhs);
StencilFn pick_f64_r9(bool ghost, int lanes, int minb, int nrhs);
StencilFn pick_f32_r9(bool ghost, int lanes, int minb, int nrhs);
StencilFn pick_mixed_r9(bool ghost, int lanes, int minb, int nrhs);

// the neighbour-staged kernel (stencil.cuh dslash_stage_kernel) of one (precision, recon): lanes 1/2
StencilFn pick_f64_r18_stage(bool ghost, int lanes, int nrhs);
StencilFn pick_f64_r12_stage(bool ghost, int lanes, int nrhs);
StencilFn pick_f32_r18_stage(bool ghost, int lanes, int nrhs);
StencilFn pick_f32_r12_stage(bool ghost, int lanes, int nrhs);
StencilFn pick_mixed_r18_stage(bool ghost, int lanes, int nrhs);
StencilFn pick_mixed_r12_stage(bool ghost, int lanes, int nrhs);
StencilFn pick_f64_r9_stage(bool ghost, int lanes, int nrhs);
StencilFn pick_f32_r9_stage(bool ghost, int lanes, int nrhs);
StencilFn pick_mixed_r9_stage(bool ghost, int lanes, int nrhs);

// the site-blocked-layout kernel (dslash_apply_multi_blocked) of one (precision, recon): interior or
// ghost-aware, lanes 1/2/4 (the handle's mapping), 1/2/4/8 right-hand sides per launch
StencilFn pick_f64_r18_vblk(bool ghost, int lanes, int nrhs);
StencilFn pick_f64_r12_vblk(bool ghost, int lanes, int nrhs);
StencilFn pick_f32_r18_vblk(bool ghost, int lanes, int nrhs);
StencilFn pick_f32_r12_vblk(bool ghost, int lanes, int nrhs);
StencilFn pick_mixed_r18_vblk(bool ghost, int lanes, int nrhs);
StencilFn pick_mixed_r12_vblk(bool ghost, int lanes, int nrhs);
StencilFn pick_f64_r9_vblk(bool ghost, int lanes, int nrhs);
StencilFn pick_f32_r9_vblk(bool ghost, int lanes, int nrhs);
StencilFn pick_mixed_r9_vblk(bool ghost, int lanes, int nrhs);

}  // namespace hisq
