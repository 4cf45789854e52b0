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

// the site-blocked layout (dslash_apply_multi_blocked): MINB 2, the handle's mapping (its link
// layout), interior or ghost-aware
template <typename LR, typename VR, int LANES, bool GHOST, int RECON>
StencilFn pick_vblk_n(int nrhs) {
    switch (nrhs) {
        case 2: return dslash_kernel<LR, VR, LANES, GHOST, 2, RECON, 2, 1, true>;
        case 4: return dslash_kernel<LR, VR, LANES, GHOST, 2, RECON, 4, 1, true>;
        case 8:
            // interior, recon 18 / 12: one thread per site holds all 8 right-hand sides; fp64 vectors
            // (f64, mixed) at 255 registers and 8 warps/SM: 355 vs 388 us for 2 groups x 4 at 32^4
            // fp64, mixed 297 vs 351 us; fp32 vectors at 128 registers and 16 warps/SM: 167 vs
            // 178 us (recon-12 161 vs 181 us).  Recon-9 (its rebuild needs the registers: 717 vs
            // 502 us) and the ghost-aware boundary kernel keep 2 groups x 4
            // (profiles/r03/blocked/).  dslash_lib.cu vblk_groups8 matches.
            if constexpr (RECON != 9 && !GHOST)
                return dslash_kernel<LR, VR, LANES, GHOST, sizeof(VR) == 8 ? 1 : 2, RECON, 8, 1, true>;
            else
                return dslash_kernel<LR, VR, LANES, GHOST, 2, RECON, 4, 2, true>;
        default: return dslash_kernel<LR, VR, LANES, GHOST, 2, RECON, 1, 1, true>;
    }
}

template <typename LR, typename VR, bool GHOST, int RECON>
StencilFn pick_vblk_l(int lanes, int nrhs) {
    return lanes == 1   ? pick_vblk_n<LR, VR, 1, GHOST, RECON>(nrhs)
           : lanes == 2 ? pick_vblk_n<LR, VR, 2, GHOST, RECON>(nrhs)
                        : pick_vblk_n<LR, VR, 4, GHOST, RECON>(nrhs);
}

template <typename LR, typename VR, int RECON>
StencilFn pick_vblk(bool ghost, int lanes, int nrhs) {
    return ghost ? pick_vblk_l<LR, VR, true, RECON>(lanes, nrhs) : pick_vblk_l<LR, VR, false, RECON>(lanes, nrhs);
}

}  // namespace hisq

#define HISQ_DEFINE_PICK(NAME, LR, VR, RECON)                                                                  \
    namespace hisq {                                                                                          \
    StencilFn NAME(bool ghost, int lanes, int minb, int nrhs) {                                               \
        return pick_any<LR, VR, RECON>(ghost, lanes, minb, nrhs);                                             \
    }                                                                                                         \
    StencilFn NAME##_stage(bool ghost, int lanes, int nrhs) { return pick_stage<LR, VR, RECON>(ghost, lanes, nrhs); } \
    StencilFn NAME##_vblk(bool ghost, int lanes, int nrhs) { return pick_vblk<LR, VR, RECON>(ghost, lanes, nrhs); } \
    }
