// dispatch.h -- kernel selection across the per-precision translation units (kernels_*.cu).
#pragma once

#include "common.cuh"

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
