// stencil.cuh -- the single-parity HISQ Dslash kernels for sm_100a.
//
// Operation (Eq. (1) + Naik terms L27/L51; include/hisq_dslash.h): for each
// target site x,  chi(x) = sum_mu [ Ff(x,mu) psi(x+mu) - Fb(x,mu) psi(x-mu)
//                                 + Nf(x,mu) psi(x+3mu) - Nb(x,mu) psi(x-3mu) ]
// where Fb(x,mu) = F(x-mu,mu)^dag and Nb(x,mu) = N(x-3mu,mu)^dag were precomputed by
// load_links (|l| = 4 link arrays).
//
// The path is HBM-bound: 16 link matrices x 144 B = 2304 B streamed once per site against
// 1146 flop; the 16 neighbour vectors are reused 16x from L1/L2.
// Links are read with L1::no_allocate + L2 evict_first, vectors with L2 evict_last, the
// output with st.global.cs.
//
// Two mappings (chosen by measurement):
//   SITE : one thread per target site (the paper's 1LP decomposition, L59-87);
//   DIR4 : four consecutive lanes per site, lane = mu, each lane streams that direction's
//          4 matrices and the partial sums meet in two __shfl_xor steps (the paper's 3LP-1
//          "site x direction + reduction" idea, L101-142, with shuffles instead of local
//          memory + barrier and without the row split, which replicates vector loads).
#pragma once

#include "common.cuh"

namespace hisq {

// Internal link layouts (double2 per complex element e = 3*i + j of a 3x3 matrix).
// l: 0 = Ff (+1 hop), 1 = Fb (-1), 2 = Nf (+3), 3 = Nb (-3).
//   SITE: links[((mu*4 + l)*9 + e) * vh + cb]       (16 x 9 coalesced streams per site block)
//   DIR4: links[((l*9 + e) * vh + cb) * 4 + mu]     (lanes 4s..4s+3 read 64 contiguous bytes)
__host__ __device__ __forceinline__ int64_t link_index_site(int mu, int l, int e, int64_t vh, int64_t cb) {
    return ((int64_t)((mu * 4 + l) * 9 + e)) * vh + cb;
}
__host__ __device__ __forceinline__ int64_t link_index_dir4(int mu, int l, int e, int64_t vh, int64_t cb) {
    return (((int64_t)(l * 9 + e)) * vh + cb) * 4 + mu;
}

struct Site {
    int x, y, z, t, xh;
    int64_t cb;
};

// thread -> target site of the box list (t slowest, so the L2 working set is a sliding window)
__device__ __forceinline__ Site decode_site(const StencilParams& P, int64_t gid) {
    int b = 0;
#pragma unroll
    for (int k = 1; k < kMaxBoxes; ++k)
        if (k < P.nbox && gid >= P.box_start[k]) b = k;
    const Box& B = P.box[b];
    uint32_t r = (uint32_t)(gid - P.box_start[b]);
    uint32_t q = P.div_xh[b].div(r);
    Site s;
    s.xh = (int)(r - q * (uint32_t)(B.n[0] >> 1)) + (B.lo[0] >> 1);
    r = q;
    q = P.div_y[b].div(r);
    s.y = (int)(r - q * (uint32_t)B.n[1]) + B.lo[1];
    r = q;
    q = P.div_z[b].div(r);
    s.z = (int)(r - q * (uint32_t)B.n[2]) + B.lo[2];
    s.t = (int)q + B.lo[3];
    s.x = 2 * s.xh + ((P.parity + s.y + s.z + s.t) & 1);
    s.cb = s.xh + (int64_t)P.lxh * (s.y + (int64_t)P.L[1] * (s.z + (int64_t)P.L[2] * s.t));
    return s;
}

struct SrcRef {
    const double2* p;  // colour component c at p[c * stride]
    int64_t stride;
};

// Address of psi(x + h mu^).  GHOST: directions in P.halo_mask read the depth-3 ghost faces
// outside [0, L); otherwise coordinates wrap periodically (two conditional steps suffice for
// |h| <= 3 and L >= 2).
template <bool GHOST>
__device__ __forceinline__ SrcRef source(const StencilParams& P, int mu, int h, const Site& s) {
    const int c = mu == 0 ? s.x : mu == 1 ? s.y : mu == 2 ? s.z : s.t;
    const int L = P.L[mu];
    int cn = c + h;
    if (GHOST && mu >= 2 && ((P.halo_mask >> mu) & 1) && (cn < 0 || cn >= L)) {
        const int side = cn >= L;
        const int d = side ? cn - L : cn + 3;
        int64_t f;
        if (mu == 3)
            f = s.xh + (int64_t)P.lxh * (s.y + (int64_t)P.L[1] * (s.z + (int64_t)P.L[2] * d));
        else
            f = s.xh + (int64_t)P.lxh * (s.y + (int64_t)P.L[1] * (d + 3 * (int64_t)s.t));
        return {P.ghost[mu][side] + f, P.face_vh[mu]};
    }
    if (cn < 0) cn += L;
    if (cn < 0) cn += L;
    if (cn >= L) cn -= L;
    if (cn >= L) cn -= L;
    int64_t idx;
    if (mu == 0) {
        idx = s.cb - s.xh + (cn >> 1);
    } else {
        const int64_t st = mu == 1 ? (int64_t)P.lxh
                         : mu == 2 ? (int64_t)P.lxh * P.L[1]
                                   : (int64_t)P.lxh * P.L[1] * P.L[2];
        idx = s.cb + (int64_t)(cn - c) * st;
    }
    return {P.in + idx, P.vh};
}

// acc (+/-)= U v for a 3x3 matrix whose 9 elements are U[e]
template <bool SUB>
__device__ __forceinline__ void matvec_acc(double2 acc[3], const double2 U[9], const double2 v[3]) {
#pragma unroll
    for (int i = 0; i < 3; ++i)
#pragma unroll
        for (int j = 0; j < 3; ++j) {
            if (SUB)
                cmsub(acc[i], U[3 * i + j], v[j]);
            else
                cmadd(acc[i], U[3 * i + j], v[j]);
        }
}

// ---------------------------------------------------------------- SITE: one thread per site
template <bool GHOST>
__global__ void __launch_bounds__(256) dslash_site_kernel(const StencilParams P) {
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (gid >= P.box_start[P.nbox]) return;
    const uint64_t pol_stream = policy_evict_first();
    const uint64_t pol_keep = policy_evict_last();
    const Site s = decode_site(P, gid);
    double2 acc[3] = {{0.0, 0.0}, {0.0, 0.0}, {0.0, 0.0}};
#pragma unroll
    for (int mu = 0; mu < 4; ++mu) {
#pragma unroll
        for (int l = 0; l < 4; ++l) {
            const int h = (l == 0) ? 1 : (l == 1) ? -1 : (l == 2) ? 3 : -3;
            const SrcRef src = source<GHOST>(P, mu, h, s);
            double2 v[3];
#pragma unroll
            for (int c = 0; c < 3; ++c) v[c] = ld_reuse(src.p + c * src.stride, pol_keep);
            const double2* lp = P.links + link_index_site(mu, l, 0, P.vh, s.cb);
            double2 U[9];
#pragma unroll
            for (int e = 0; e < 9; ++e) U[e] = ld_stream(lp + (int64_t)e * P.vh, pol_stream);
            if (l & 1)
                matvec_acc<true>(acc, U, v);
            else
                matvec_acc<false>(acc, U, v);
        }
    }
#pragma unroll
    for (int c = 0; c < 3; ++c) st_stream(P.out + c * P.vh + s.cb, acc[c]);
}

// ---------------------------------------------------------------- DIR4: four lanes per site
template <bool GHOST>
__global__ void __launch_bounds__(256) dslash_dir4_kernel(const StencilParams P) {
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int mu = threadIdx.x & 3;
    const int64_t site = gid >> 2;
    const bool valid = site < P.box_start[P.nbox];
    double2 acc[3] = {{0.0, 0.0}, {0.0, 0.0}, {0.0, 0.0}};
    Site s;
    if (valid) {
        const uint64_t pol_stream = policy_evict_first();
        const uint64_t pol_keep = policy_evict_last();
        s = decode_site(P, site);
#pragma unroll
        for (int l = 0; l < 4; ++l) {
            const int h = (l == 0) ? 1 : (l == 1) ? -1 : (l == 2) ? 3 : -3;
            const SrcRef src = source<GHOST>(P, mu, h, s);
            double2 v[3];
#pragma unroll
            for (int c = 0; c < 3; ++c) v[c] = ld_reuse(src.p + c * src.stride, pol_keep);
            const double2* lp = P.links + link_index_dir4(mu, l, 0, P.vh, s.cb);
            double2 U[9];
#pragma unroll
            for (int e = 0; e < 9; ++e) U[e] = ld_stream(lp + (int64_t)e * P.vh * 4, pol_stream);
            if (l & 1)
                matvec_acc<true>(acc, U, v);
            else
                matvec_acc<false>(acc, U, v);
        }
    }
    // butterfly over the 4 lanes of a site: every lane ends with ((p0+p1)+(p2+p3)) bitwise
#pragma unroll
    for (int c = 0; c < 3; ++c) {
#pragma unroll
        for (int off = 1; off <= 2; off <<= 1) {
            acc[c].x += __shfl_xor_sync(0xffffffffu, acc[c].x, off);
            acc[c].y += __shfl_xor_sync(0xffffffffu, acc[c].y, off);
        }
    }
    if (valid && mu < 3) {
        const double2 r = mu == 0 ? acc[0] : mu == 1 ? acc[1] : acc[2];
        st_stream(P.out + mu * P.vh + s.cb, r);
    }
}

}  // namespace hisq
