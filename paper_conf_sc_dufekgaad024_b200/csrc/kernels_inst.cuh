// kernels_inst.cuh -- instantiation table of dslash_kernel for one (LR, VR, RECON); included by
// the kernels_*.cu translation units, which build in parallel.
// Instantiated: every (lanes, ghost) with MINB 2/3/4 for one right-hand side, with MINB 2
// (the measured best) for 2 and 4 right-hand sides per launch; 8 right-hand sides run as two
// adjacent thread groups of 4 register-blocked ones (8 per thread needs 255 registers and ran at
// 12% occupancy).
#pragma once

#include "dispatch.h"
#include "stencil.cuh"

namespace hisq {

template <typename LR, typename VR, int LANES, bool GHOST, int RECON>
StencilFn pick_minb(int minb, int nrhs) {
    switch (nrhs) {
        case 2: return dslash_kernel<LR, VR, LANES, GHOST, 2, RECON, 2>;
        case 4: return dslash_kernel<LR, VR, LANES, GHOST, 2, RECON, 4>;
        case 8: return dslash_kernel<LR, VR, LANES, GHOST, 2, RECON, 4, 2>;  // 2 thread groups x 4 RHS each
        default: break;
    }
    switch (minb) {
        case 2: return dslash_kernel<LR, VR, LANES, GHOST, 2, RECON>;
        case 3: return dslash_kernel<LR, VR, LANES, GHOST, 3, RECON>;
        default: return dslash_kernel<LR, VR, LANES, GHOST, 4, RECON>;
    }
}

template <typename LR, typename VR, bool GHOST, int RECON>
StencilFn pick_lanes(int lanes, int minb, int nrhs) {
    switch (lanes) {
        case 1: return pick_minb<LR, VR, 1, GHOST, RECON>(minb, nrhs);
        case 2: return pick_minb<LR, VR, 2, GHOST, RECON>(minb, nrhs);
        default: return pick_minb<LR, VR, 4, GHOST, RECON>(minb, nrhs);
    }
}

template <typename LR, typename VR, int RECON>
StencilFn pick_any(bool ghost, int lanes, int minb, int nrhs) {
    return ghost ? pick_lanes<LR, VR, true, RECON>(lanes, minb, nrhs) : pick_lanes<LR, VR, false, RECON>(lanes, minb, nrhs);
}

// the neighbour-staged kernel (DSLASH_OPT_STAGE): LANES 1 and 2, MINB 2, 1/2/4/8 right-hand sides
template <typename LR, typename VR, int LANES, bool GHOST, int RECON>
StencilFn pick_stage_n(int nrhs) {
    switch (nrhs) {
        case 2: return dslash_stage_kernel<LR, VR, LANES, GHOST, RECON, 2>;
        case 4: return dslash_stage_kernel<LR, VR, LANES, GHOST, RECON, 4>;
        case 8: return dslash_stage_kernel<LR, VR, LANES, GHOST, RECON, 4, 2>;
        default: return dslash_stage_kernel<LR, VR, LANES, GHOST, RECON, 1>;
    }
}

template <typename LR, typename VR, int RECON>
StencilFn pick_stage(bool ghost, int lanes, int nrhs) {
    if (lanes == 1)
        return ghost ? pick_stage_n<LR, VR, 1, true, RECON>(nrhs) : pick_stage_n<LR, VR, 1, false, RECON>(nrhs);
    return ghost ? pick_stage_n<LR, VR, 2, true, RECON>(nrhs) : pick_stage_n<LR, VR, 2, false, RECON>(nrhs);
}

// the one-shot fused kernel (DSLASH_OVERLAP_FUSED): main launch or clean-up, lanes 1/2/4
template <typename LR, typename VR, int RECON>
FusedFn pick_fused(bool cleanup, int lanes) {
    switch (lanes) {
        case 1: return cleanup ? dslash_fused_cleanup<LR, VR, 1, RECON> : dslash_fused_kernel<LR, VR, 1, RECON>;
        case 2: return cleanup ? dslash_fused_cleanup<LR, VR, 2, RECON> : dslash_fused_kernel<LR, VR, 2, RECON>;
        default: return cleanup ? dslash_fused_cleanup<LR, VR, 4, RECON> : dslash_fused_kernel<LR, VR, 4, RECON>;
    }
}

template <typename LR, typename VR, int LANES, int RECON>
PersistFn pick_persist_l(int mode) {
    switch (mode) {
        case 0: return dslash_persistent_kernel<LR, VR, LANES, false, RECON, false>;  // no halo
        case 1: return dslash_persistent_kernel<LR, VR, LANES, true, RECON, false>;   // halo, main
        default: return dslash_persistent_kernel<LR, VR, LANES, true, RECON, true>;   // halo, clean-up
    }
}

template <typename LR, typename VR, int RECON>
PersistFn pick_persist(int mode, int lanes) {
    switch (lanes) {
        case 1: return pick_persist_l<LR, VR, 1, RECON>(mode);
        case 2: return pick_persist_l<LR, VR, 2, RECON>(mode);
        default: return pick_persist_l<LR, VR, 4, RECON>(mode);
    }
}

}  // namespace hisq

#define HISQ_DEFINE_PICK(NAME, PNAME, LR, VR, RECON)                           \
    namespace hisq {                                                           \
    StencilFn NAME(bool ghost, int lanes, int minb, int nrhs) {                \
        return pick_any<LR, VR, RECON>(ghost, lanes, minb, nrhs);              \
    }                                                                          \
    PersistFn PNAME(int mode, int lanes) { return pick_persist<LR, VR, RECON>(mode, lanes); } \
    StencilFn NAME##_stage(bool ghost, int lanes, int nrhs) { return pick_stage<LR, VR, RECON>(ghost, lanes, nrhs); } \
    FusedFn NAME##_fused(bool cleanup, int lanes) { return pick_fused<LR, VR, RECON>(cleanup, lanes); } \
    }
