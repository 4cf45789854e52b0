// dispatch.h -- kernel selection across the per-precision translation units (kernels_*.cu).
#pragma once

#include "common.cuh"
#include "stencil.cuh"

namespace hisq {

typedef void (*StencilFn)(StencilParams);

typedef void (*PersistFn)(StencilParams, PersistArgs);

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

// the one-shot fused kernel (stencil.cuh dslash_fused_kernel / _cleanup) of one (precision, recon)
typedef void (*FusedFn)(StencilParams, FusedArgs);
FusedFn pick_f64_r18_fused(bool cleanup, int lanes);
FusedFn pick_f64_r12_fused(bool cleanup, int lanes);
FusedFn pick_f32_r18_fused(bool cleanup, int lanes);
FusedFn pick_f32_r12_fused(bool cleanup, int lanes);
FusedFn pick_mixed_r18_fused(bool cleanup, int lanes);
FusedFn pick_mixed_r12_fused(bool cleanup, int lanes);
FusedFn pick_f64_r9_fused(bool cleanup, int lanes);
FusedFn pick_f32_r9_fused(bool cleanup, int lanes);
FusedFn pick_mixed_r9_fused(bool cleanup, int lanes);

// the persistent fused kernel (stencil.cuh) of one (precision, recon): lanes 1/2/4; mode 0 = no
// halo, 1 = halo (interior, then boundary tiles if the faces have landed), 2 = boundary clean-up
PersistFn persist_f64_r18(int mode, int lanes);
PersistFn persist_f64_r12(int mode, int lanes);
PersistFn persist_f32_r18(int mode, int lanes);
PersistFn persist_f32_r12(int mode, int lanes);
PersistFn persist_mixed_r18(int mode, int lanes);
PersistFn persist_mixed_r12(int mode, int lanes);
PersistFn persist_f64_r9(int mode, int lanes);
PersistFn persist_f32_r9(int mode, int lanes);
PersistFn persist_mixed_r9(int mode, int lanes);

// The TMA-staged persistent kernel (bulk.cuh): function, dynamic shared memory, threads per CTA,
// sites per tile.  precision: 0 fp64, 1 fp32, 2 mixed (DSLASH_F64/F32/MIXED).
typedef void (*BulkFn)(StencilParams, unsigned long long*, unsigned long long);
struct BulkKernel {
    BulkFn fn;
    size_t smem;
    int threads;
    int tile;
    int batch;  // tiles per scheduler draw
};
BulkKernel pick_bulk(int precision, int recon, bool ghost);

}  // namespace hisq
