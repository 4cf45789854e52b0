// rhs8_tma.cuh -- 8 right-hand sides with a TMA-fed link pipeline (fp64, full long links, the
// SITE link layout).  SURVEY.md §8(f)-4: one link pass serves 8 vectors (the L25 intensity
// argument), 3072 B/site against 8 x 1146 flop.
//
// Why (profiles/r02/mrhs/): the register-blocked 8-RHS kernel (2 thread groups x 4 RHS) is
// latency-bound.  A hop needs 9 link loads that miss to DRAM plus 12 neighbour loads that mostly
// hit L2, and under the 128-register budget the compiler cannot keep the next hop's loads in flight,
// so every hop waits ~one DRAM round trip.  Here the links never touch the registers or the
// warps' critical path: each warp streams its tile's 16 link matrices through a 4-deep ring of
// shared-memory stages with cp.async.bulk.tensor (the TMA engine, SASS UTMALDG) and mbarrier
// completion, a hop ahead by 4, while the warp only gathers neighbours from L2.
//
// Mapping: as the register kernel's quarter-warp runs -- a warp owns a tile of 16 consecutive
// target sites, lanes (l >> 4) * 8 + (l & 7) are its site and (l >> 3) & 1 its right-hand-side
// group (4 RHS each).  The two groups of a site read the same link entries from shared memory
// (broadcast).  Per (site, rhs) the summation order is the register kernel's (mu, l, row, column),
// so the results are bitwise those of the single-RHS apply.
//
// Tensor map (host, dslash_lib.cu): the SITE link array of one parity viewed as a 3-D tensor of
// doubles [entry 36][mu 4][2 vh], entry = base(l) + e; one box = 9 entries (one matrix) x 1 mu
// x 16 sites = 2304 B, landing in shared memory as [e][site] complex.
#pragma once

#include <cuda.h>

#include "common.cuh"
#include "dispatch.h"
#include "stencil.cuh"

namespace hisq {

constexpr int kRhs8Stages = 4;  // ring depth per warp (a hop every 4 ahead)

// NRHS right-hand sides per thread, RHSL = 8 / NRHS thread groups per site (quarter-warp runs of
// 8 sites), TS = 32 / RHSL sites per warp tile; WARPS per CTA, MINB CTAs per SM
template <int NRHS>
struct Rhs8Cfg {
    static constexpr int RHSL = 8 / NRHS;
    static constexpr int TS = 32 / RHSL;
    static constexpr uint32_t kStage = 9 * TS * 16;  // one matrix of the tile
    static constexpr int WARPS = NRHS == 4 ? 8 : 8;
    static constexpr int MINB = NRHS == 4 ? 2 : 3;
    static constexpr size_t smem() { return (size_t)WARPS * kRhs8Stages * (kStage + 8); }
};

// ld_reuse that keeps its place among the other volatile asm of the kernel
__device__ __forceinline__ double2 ld_reuse_ordered(const double2* p, uint64_t pol) {
    double2 r;
    asm volatile("ld.global.nc.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;" : "=d"(r.x), "=d"(r.y) : "l"(p), "l"(pol));
    return r;
}

__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, int c0, int c1, int c2, uint64_t* bar,
                                            uint64_t pol) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%2, %3, %4}], [%5], %6;" ::"r"(smem_addr(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_addr(bar)), "l"(pol)
        : "memory");
}

// P: the full-lattice box (enumeration order = cb order), vh a multiple of the tile; in/out hold
// 8 vectors [8][3][vh].
template <int UNROLL, int NRHS>
__global__ void __launch_bounds__(32 * Rhs8Cfg<NRHS>::WARPS, Rhs8Cfg<NRHS>::MINB)
    dslash_rhs8_tma_kernel(const __grid_constant__ CUtensorMap tmap, const StencilParams P) {
    using V2 = double2;
    using C = Rhs8Cfg<NRHS>;
    constexpr int TS = C::TS;
    constexpr uint32_t kStageB = C::kStage;
    asm volatile("griddepcontrol.launch_dependents;");
    extern __shared__ __align__(128) unsigned char smem[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned char* ring = smem + (size_t)warp * kRhs8Stages * kStageB;
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + (size_t)C::WARPS * kRhs8Stages * kStageB) + warp * kRhs8Stages;
    const int64_t ntiles = P.vh / TS;
    const int64_t nw = (int64_t)gridDim.x * C::WARPS;
    int64_t tile = (int64_t)blockIdx.x * C::WARPS + warp;
    const uint64_t pol_first = policy_evict_first();
    const uint64_t pol_keep = policy_evict_last();
    if (lane == 0) {
        for (int k = 0; k < kRhs8Stages; ++k) mbar_init(&full[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    // hop j = 4 mu + l of a tile lives in stage j & 3 with phase (j >> 2) & 1 (4 uses per tile)
    auto issue = [&](int64_t t, int j) {  // lane 0
        uint64_t* bar = &full[j & 3];
        mbar_arrive_expect_tx(bar, kStageB);
        tma_load_3d(ring + (j & 3) * kStageB, &tmap, (int)(2 * t * TS), j >> 2, 9 * (j & 3), bar, pol_first);
    };
    // links are read-only: the first tile's first 4 matrices are requested before the PDL wait
    if (lane == 0 && tile < ntiles)
        for (int j = 0; j < kRhs8Stages; ++j) issue(tile, j);
    const void* in;
    asm volatile("griddepcontrol.wait;\n\tmov.b64 %0, %1;" : "=l"(in) : "l"(P.in) : "memory");
    const int rl = (lane >> 3) % C::RHSL;                       // right-hand-side group
    const int sl = ((lane >> 3) / C::RHSL) * 8 + (lane & 7);    // site in the tile
    for (; tile < ntiles; tile += nw) {
        const Site s = decode_site(P, tile * TS + sl);
        V2 acc[NRHS][3];
#pragma unroll
        for (int r = 0; r < NRHS; ++r)
#pragma unroll
            for (int c = 0; c < 3; ++c) acc[r][c].x = acc[r][c].y = 0.0;
        // unrolled by direction (the 4 hops of a direction: l known at compile time, mu at run
        // time); the neighbour loads are volatile asm (ld_reuse_ordered), so the compiler cannot
        // hoist later hops' loads above this hop's shared-memory reads (fully unrolled and hoisted,
        // the kernel spilled 3.5 KB)
#pragma unroll UNROLL
        for (int j = 0; j < 16; ++j) {
            const int mu = j >> 2, l = j & 3;
            const int h = (l == 0) ? 1 : (l == 1) ? -1 : (l == 2) ? 3 : -3;
            const SrcRef<V2> src = source<V2, false>(P, in, mu, h, s, rl * NRHS);
            V2 v[NRHS][3];
#pragma unroll
            for (int r = 0; r < NRHS; ++r)
#pragma unroll
                for (int c = 0; c < 3; ++c)
                    v[r][c] = ld_reuse_ordered(src.p + (int64_t)r * 3 * src.stride + c * src.stride, pol_keep);
            mbar_wait(&full[j & 3], (j >> 2) & 1);
            const V2* st = reinterpret_cast<const V2*>(ring + (j & 3) * kStageB);
            // entry by entry from shared memory (4 registers, not a 36-register matrix), each applied
            // to the 4 right-hand sides; acc[r][i] receives columns j = 0, 1, 2 in order, as in
            // matvec_acc
#pragma unroll
            for (int e = 0; e < 9; ++e) {
                const V2 u = lds(st + e * TS + sl);
#pragma unroll
                for (int r = 0; r < NRHS; ++r) {
                    if (l & 1)
                        cmsub(acc[r][e / 3], u, v[r][e % 3]);
                    else
                        cmadd(acc[r][e / 3], u, v[r][e % 3]);
                }
            }
            __syncwarp();  // every lane has read the stage: it may be refilled
            if (lane == 0) {
                // the lanes' generic-proxy reads of the stage precede the TMA (async-proxy) refill
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                if (j + kRhs8Stages < 16)
                    issue(tile, j + kRhs8Stages);
                else if (tile + nw < ntiles)
                    issue(tile + nw, j + kRhs8Stages - 16);
            }
        }
#pragma unroll
        for (int r = 0; r < NRHS; ++r) {
            V2* out = static_cast<V2*>(P.out) + (int64_t)(rl * NRHS + r) * 3 * P.vh;
#pragma unroll
            for (int c = 0; c < 3; ++c) st_stream(out + c * P.vh + s.cb, acc[r][c]);
        }
    }
}

}  // namespace hisq
