// stencil_mrhs.cuh -- the 8-right-hand-side stencil with the link stream on the TMA engine.
//
// Same operation, thread mapping and summation order as dslash_kernel<double, double, 1, false,
// 2, RECON, 4, 2> (stencil.cuh): one thread per (site, group of 4 right-hand sides), the two
// groups of a site in quarter-warp runs of 8 sites (a warp = 16 sites x 2 groups), the 16 hops in
// the order mu = 0..3, l = Ff, Fb, Nf, Nb, and per (site, rhs) the same FMA sequence
// (matvec_acc), so the results are bitwise those of the plain kernel.
//
// What differs is where the link matrices travel.  The plain kernel loads them into registers
// (9 x 16 B per thread and hop, DRAM latency) through the same L1 miss path as the neighbour
// gathers; round 3 measured that the two streams then ADD UP instead of overlapping (links alone
// 241 us, gathers alone 156 us, both 342-353 us without any arithmetic; profiles/r03/mrhs/).
// Here each warp streams its 16 sites' link matrices through a ring of S shared-memory stages
// with cp.async.bulk (the TMA engine: no registers, no L1 miss slots), D hops ahead, one bulk copy
// of 16 x 16 B per matrix entry (the warp's 16 sites are 16 consecutive target sites, and entry e
// of a matrix is one contiguous span over sites in the link layout), completing on the stage's
// mbarrier.  The threads read the matrix from shared memory when they multiply; the register
// file is left to the neighbour gathers.  Used for interior launches whose box enumerates
// consecutive sites in 16-site runs (full x, y and z extents; dslash_lib.cu rhs8_tma_ok).
#pragma once

#include "stencil.cuh"

namespace hisq {

constexpr int kTmaWarps = 8;          // 256-thread blocks
constexpr int kTmaEntryBytes = 256;   // one matrix entry (16 B) of the warp's 16 sites
constexpr int kTmaStageBytes = 9 * kTmaEntryBytes;

// wait for phase `parity` of the stage's mbarrier; returns sbase from inside the waiting asm
__device__ __forceinline__ uint32_t stage_wait_parity(uint64_t* bar, uint32_t parity, uint32_t sbase) {
    uint32_t b;
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "TWAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "@!p bra TWAIT_%=;\n\t"
        "mov.b32 %0, %3;\n}"
        : "=r"(b)
        : "r"(smem_addr(bar)), "r"(parity), "r"(sbase)
        : "memory");
    return b;
}

template <int S>
constexpr size_t rhs8_tma_smem() {
    return (size_t)kTmaWarps * S * kTmaStageBytes;
}

template <int RECON, int S, int D>
__global__ void __launch_bounds__(256, 2) dslash_rhs8_tma_kernel(const StencilParams P) {
    static_assert(RECON == 18 || RECON == 12, "fp64 links, recon 18 / 12");
    static_assert(D >= 1 && D < S, "prefetch distance");
    using V2 = double2;
    constexpr int kHops = 16, NRHS = 4;
    extern __shared__ __align__(128) unsigned char tma_smem[];
    __shared__ uint64_t bars[kTmaWarps][S];
    asm volatile("griddepcontrol.launch_dependents;");

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int rl = (int)((gid >> 3) & 1);                   // right-hand-side group
    const int siw = ((lane >> 4) << 3) | (lane & 7);        // site within the warp's 16
    const int64_t site = (gid >> 5) * 16 + siw;
    if ((gid >> 5) * 16 >= P.box_start[P.nbox]) return;     // whole warps (sites % 16 == 0)
    const uint64_t pol_stream = policy_evict_first();
    const uint64_t pol_keep = policy_evict_last();
    const Site s = decode_site(P, site);
    const int64_t cb0 = s.cb - siw;                         // first site of the warp's run
    const double2* links = static_cast<const double2*>(P.links);
    unsigned char* ring = tma_smem + (size_t)warp * S * kTmaStageBytes;
    uint64_t* bar = bars[warp];
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < S; ++k) mbar_init(&bar[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();

    // lanes 0 .. elems-1 each copy one entry of hop q's matrix (16 sites x 16 B) into stage q % S
    auto issue = [&](int q) {
        const int mu = q >> 2, l = q & 3, st = q % S;
        const int ne = elems_of<RECON>(l);
        if (lane == 0) mbar_arrive_expect_tx(&bar[st], (uint32_t)(ne * kTmaEntryBytes));
        __syncwarp();
        if (lane < ne)
            bulk_g2s(ring + st * kTmaStageBytes + lane * kTmaEntryBytes,
                     links + link_index<1, RECON>(mu, l, lane, P.vh, cb0), kTmaEntryBytes, &bar[st], pol_stream);
    };

    V2 acc[NRHS][3];
#pragma unroll
    for (int r = 0; r < NRHS; ++r)
#pragma unroll
        for (int c = 0; c < 3; ++c) acc[r][c].x = acc[r][c].y = 0.0;

    // links are read-only: the first D matrices are requested before the PDL wait
#pragma unroll
    for (int q = 0; q < D; ++q) issue(q);
    const void* in;
    asm volatile("griddepcontrol.wait;\n\tmov.b64 %0, %1;" : "=l"(in) : "l"(P.in) : "memory");

#pragma unroll
    for (int q = 0; q < kHops; ++q) {
        const int mu = q >> 2, l = q & 3, h = (l == 0) ? 1 : (l == 1) ? -1 : (l == 2) ? 3 : -3;
        if (q + D < kHops) {
            // stage (q + D) % S was last read at hop q + D - S < q: every lane is past it
            __syncwarp();
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            issue(q + D);
        }
        const SrcRef<V2> src = source<V2, false>(P, in, mu, h, s, rl * NRHS);
        V2 v[NRHS][3];
#pragma unroll
        for (int r = 0; r < NRHS; ++r)
#pragma unroll
            for (int c = 0; c < 3; ++c)
                v[r][c] = (kZtNoL1 && mu >= 2) ? ld_reuse_na(src.p + (int64_t)(r * 3 + c) * src.stride, pol_keep)
                                               : ld_reuse(src.p + (int64_t)(r * 3 + c) * src.stride, pol_keep);
        // the stage's bytes have landed; the returned address comes out of the waiting asm, so no
        // shared load of the matrix is scheduled above the wait
        const uint32_t sa = stage_wait_parity(&bar[q % S], (uint32_t)((q / S) & 1),
                                              smem_addr(ring + (q % S) * kTmaStageBytes)) +
                            (uint32_t)siw * 16u;
        V2 U[9];
#pragma unroll
        for (int e = 0; e < elems_of<RECON>(l); ++e) U[e] = lds_at(sa + (uint32_t)(e * kTmaEntryBytes), (V2*)nullptr);
        if (elems_of<RECON>(l) == 6) reconstruct_row2(U, P.long_inv_scale);
#pragma unroll
        for (int r = 0; r < NRHS; ++r) {
            if (l & 1)
                matvec_acc<true>(acc[r], U, v[r]);
            else
                matvec_acc<false>(acc[r], U, v[r]);
        }
    }
#pragma unroll
    for (int r = 0; r < NRHS; ++r) {
        V2* out = static_cast<V2*>(P.out) + (int64_t)(rl * NRHS + r) * 3 * P.vh;
#pragma unroll
        for (int c = 0; c < 3; ++c) st_stream(out + c * P.vh + s.cb, acc[r][c]);
    }
}

}  // namespace hisq
