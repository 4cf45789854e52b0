// stencil_mrhs.cuh -- the multi-right-hand-side stencil with an explicit register pipeline.
//
// Same operation, mapping and summation order as dslash_kernel<LR, VR, 1, false, MINB, RECON,
// NRHS, RHSL> (stencil.cuh): one thread per (site, group of NRHS right-hand sides), RHSL groups
// per site in quarter-warp runs of 8 sites, the 16 hops in the order mu = 0..3, l = Ff, Fb, Nf, Nb,
// and per (site, rhs) the same FMA sequence (matvec_acc), so results are bitwise those of the
// plain kernel.  What differs is the schedule: the loads of hop q + LD (link) and q + VD
// (neighbour vectors) are issued into their own register buffers before hop q is multiplied, so
// a full hop of memory traffic is always in flight per thread instead of whatever the register
// budget left the compiler (the plain kernel ran its 8-RHS hops in ~3 load rounds, each a full
// L2 / DRAM latency; profiles/r02/mrhs/).  Interior (non-ghost) launches with fp64-layout links.
#pragma once

#include "stencil.cuh"

#ifndef HISQ_MRHS_NOMATH
#define HISQ_MRHS_NOMATH 0  // 1: loads only; 2: vector loads only; 3: link loads only
#endif

namespace hisq {

template <typename LR, typename VR, int RECON, int NRHS, int RHSL, int MINB, int LD, int VD>
__global__ void __launch_bounds__(256, MINB) dslash_mrhs_kernel(const StencilParams P) {
    static_assert(sizeof(LR) == 8 && RECON != 9, "fp64-layout links, recon 18 / 12");
    static_assert(LD >= 1 && LD <= 2 && VD >= 0 && VD <= 1, "pipeline depths");
    using L2 = cplx_t<LR>;
    using V2 = cplx_t<VR>;
    constexpr int kHops = 16;
    asm volatile("griddepcontrol.launch_dependents;");
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int rl = (RHSL == 1) ? 0 : (int)((gid >> 3) % RHSL);
    const int64_t site = (RHSL == 1) ? gid : (gid >> 5) * (32 / RHSL) + ((gid >> 3) / RHSL) % (4 / RHSL) * 8 + (gid & 7);
    if (site >= P.box_start[P.nbox]) return;
    const uint64_t pol_stream = policy_evict_first();
    const uint64_t pol_keep = policy_evict_last();
    const Site s = decode_site(P, site);
    const L2* links = static_cast<const L2*>(P.links);

    V2 U[LD + 1][9];
    V2 v[VD + 1][NRHS][3];
    V2 acc[NRHS][3];
#pragma unroll
    for (int r = 0; r < NRHS; ++r)
#pragma unroll
        for (int c = 0; c < 3; ++c) acc[r][c].x = acc[r][c].y = VR(0);

    auto hop_of = [](int l) { return (l == 0) ? 1 : (l == 1) ? -1 : (l == 2) ? 3 : -3; };
    auto load_links = [&](V2 (&Ub)[9], int q) {
        const int mu = q >> 2, l = q & 3;
        const L2* lp = links + link_index<1, RECON>(mu, l, 0, P.vh, s.cb);
#pragma unroll
        for (int e = 0; e < elems_of<RECON>(l); ++e)
            Ub[e] = to_cplx<V2>(widen(ld_stream(lp + (int64_t)e * 4 * P.vh, pol_stream)));
    };
    const void* in = nullptr;
    auto load_vecs = [&](V2 (&vb)[NRHS][3], int q) {
        const int mu = q >> 2, l = q & 3;
        const SrcRef<V2> src = source<V2, false>(P, in, mu, hop_of(l), s, rl * NRHS);
#pragma unroll
        for (int r = 0; r < NRHS; ++r)
#pragma unroll
            for (int c = 0; c < 3; ++c)
                vb[r][c] = (kZtNoL1 && mu >= 2) ? ld_reuse_na(src.p + (int64_t)(r * 3 + c) * src.stride, pol_keep)
                                                : ld_reuse(src.p + (int64_t)(r * 3 + c) * src.stride, pol_keep);
    };

    // prologue: the first LD link matrices before the PDL wait (links are read-only), then the
    // first VD neighbour sets
#pragma unroll
    for (int q = 0; q < LD; ++q) load_links(U[q], q);
    asm volatile("griddepcontrol.wait;\n\tmov.b64 %0, %1;" : "=l"(in) : "l"(P.in) : "memory");
#pragma unroll
    for (int q = 0; q < VD; ++q) load_vecs(v[q], q);

#pragma unroll
    for (int q = 0; q < kHops; ++q) {
        if (q + LD < kHops && HISQ_MRHS_NOMATH != 2) load_links(U[(q + LD) % (LD + 1)], q + LD);
        if (q + VD < kHops && HISQ_MRHS_NOMATH != 3) load_vecs(v[(q + VD) % (VD + 1)], q + VD);
        V2(&Uq)[9] = U[q % (LD + 1)];
        const int l = q & 3;
#if HISQ_MRHS_NOMATH
        if (HISQ_MRHS_NOMATH == 2 && q == 0)
#pragma unroll
            for (int e = 0; e < 9; ++e) Uq[e].x = Uq[e].y = VR(0);
        if (HISQ_MRHS_NOMATH == 3 && q == 0)
#pragma unroll
            for (int r = 0; r < NRHS; ++r)
#pragma unroll
                for (int c = 0; c < 3; ++c) v[0][r][c].x = v[0][r][c].y = VR(0);
        // measurement aid: the loads without the matrix arithmetic (every loaded word is consumed)
#pragma unroll
        for (int e = 0; e < elems_of<RECON>(l); ++e) acc[0][0].x += Uq[e].x + Uq[e].y;
#pragma unroll
        for (int r = 0; r < NRHS; ++r)
#pragma unroll
            for (int c = 0; c < 3; ++c) acc[r][c].y += v[q % (VD + 1)][r][c].x + v[q % (VD + 1)][r][c].y;
        continue;
#endif
        if (elems_of<RECON>(l) == 6) reconstruct_row2(Uq, (VR)P.long_inv_scale);
#pragma unroll
        for (int r = 0; r < NRHS; ++r) {
            if (l & 1)
                matvec_acc<true>(acc[r], Uq, v[q % (VD + 1)][r]);
            else
                matvec_acc<false>(acc[r], Uq, v[q % (VD + 1)][r]);
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
