// links.cuh -- one-time link preprocessing for dslash_load_links (not on the timed path).
//
// Canonical input: forward links [t][z][y][x][mu][3][3] complex over the local
// volume.  Output: for target parity p the |l| = 4 link arrays of PAPER.md L51 indexed by the
// target site (Fig. 1 caption L67: "each target site s* has |l| x |k| SU(3) matrices"):
//   Ff(x,mu) = F(x,mu),  Fb(x,mu) = F(x-mu,mu)^dag,  Nf(x,mu) = N(x,mu),  Nb(x,mu) = N(x-3mu,mu)^dag
// (reading Z2: back-links are adjoints of the neighbours' forward links).
// In a halo direction the sites x-mu / x-3mu below the local volume come from `slab[mu]`, the
// 3 coordinate slices just below the local origin received from the minus neighbour, stored
// like the canonical array with that coordinate restricted to d = 0..2 (global coordinate
// origin - 3 + d):  t: [d][z][y][x][mu][9],  z: [t][d][y][x][mu][9].
#pragma once

#include "common.cuh"
#include "stencil.cuh"

namespace hisq {

struct LinkConvParams {
    const double2* fat;           // canonical local [lex][4][9]
    const double2* lng;
    const double2* slab_fat[4];   // lower link slabs (halo directions only), see above
    const double2* slab_lng[4];
    void* links;                  // internal layout: double2 (fp64) or float2 (fp32 / mixed)
    int64_t vh;
    int L[4];
    int lxh;
    int parity;
    int halo_mask;
    int lanes;                    // layout of the kernel that will read the links: 1, 2 or 4
    int recon;                    // 18 = full matrices, 12 = long links keep rows 0 and 1 only,
                                  // 9 = long links as 8 SU(3) parameters + a phase (stencil.cuh)
    double s9;                    // recon-9: the long links' real scale s
    int paired;                   // 1: fp32 paired layout (link_index_paired), register kernels only
};

// float2 offset of entry (mu, l, e) of site cb in the layout selected by P
__host__ __device__ __forceinline__ int64_t conv_index(const LinkConvParams& P, int mu, int l, int e, int64_t cb) {
    if (P.paired) {
        const int64_t o4 = P.lanes == 1   ? link_index_paired<1>(mu, l >> 1, e, P.vh, cb)
                           : P.lanes == 2 ? link_index_paired<2>(mu, l >> 1, e, P.vh, cb)
                                          : link_index_paired<4>(mu, l >> 1, e, P.vh, cb);
        return o4 * 2 + (l & 1);
    }
    if (P.recon == 12)
        return P.lanes == 1 ? link_index<1, 12>(mu, l, e, P.vh, cb)
             : P.lanes == 2 ? link_index<2, 12>(mu, l, e, P.vh, cb)
                            : link_index<4, 12>(mu, l, e, P.vh, cb);
    if (P.recon == 9)
        return P.lanes == 1 ? link_index<1, 9>(mu, l, e, P.vh, cb)
             : P.lanes == 2 ? link_index<2, 9>(mu, l, e, P.vh, cb)
                            : link_index<4, 9>(mu, l, e, P.vh, cb);
    return P.lanes == 1 ? link_index<1>(mu, l, e, P.vh, cb)
         : P.lanes == 2 ? link_index<2>(mu, l, e, P.vh, cb)
                        : link_index<4>(mu, l, e, P.vh, cb);
}

__device__ __forceinline__ const double2* canon_link(const LinkConvParams& P, bool is_long, int mu, int x, int y,
                                                     int z, int t, int back) {
    // the link of kind (fat/long) and direction mu at site (x,y,z,t) - back * mu^
    int c[4] = {x, y, z, t};
    int cn = c[mu] - back;
    if (((P.halo_mask >> mu) & 1) && cn < 0) {
        const int d = cn + 3;
        int64_t off;
        if (mu == 3)
            off = x + (int64_t)P.L[0] * (y + (int64_t)P.L[1] * (z + (int64_t)P.L[2] * d));
        else  // mu == 2
            off = x + (int64_t)P.L[0] * (y + (int64_t)P.L[1] * (d + 3 * (int64_t)t));
        return (is_long ? P.slab_lng[mu] : P.slab_fat[mu]) + (off * 4 + mu) * 9;
    }
    while (cn < 0) cn += P.L[mu];
    c[mu] = cn;
    const int64_t lex = c[0] + (int64_t)P.L[0] * (c[1] + (int64_t)P.L[1] * (c[2] + (int64_t)P.L[2] * c[3]));
    return (is_long ? P.lng : P.fat) + (lex * 4 + mu) * 9;
}

// recon-9 compression of M = s e^{i psi} W (stencil.cuh reconstruct_9): psi = arg(det M) / 3,
// W = e^{-i psi} M / s; P[0] = (arg W00, arg W20) / pi, P[1] = W01, P[2] = W02, P[3] = W10; the
// returned psi is in units of pi too
__device__ __forceinline__ void compress_9(const double2 M[9], double s, double2 P[4], double& psi) {
    const double2 m0 = make_double2(M[4].x * M[8].x - M[4].y * M[8].y - (M[5].x * M[7].x - M[5].y * M[7].y),
                                    M[4].x * M[8].y + M[4].y * M[8].x - (M[5].x * M[7].y + M[5].y * M[7].x));
    const double2 m1 = make_double2(M[3].x * M[8].x - M[3].y * M[8].y - (M[5].x * M[6].x - M[5].y * M[6].y),
                                    M[3].x * M[8].y + M[3].y * M[8].x - (M[5].x * M[6].y + M[5].y * M[6].x));
    const double2 m2 = make_double2(M[3].x * M[7].x - M[3].y * M[7].y - (M[4].x * M[6].x - M[4].y * M[6].y),
                                    M[3].x * M[7].y + M[3].y * M[7].x - (M[4].x * M[6].y + M[4].y * M[6].x));
    const double2 d0 = cmul(M[0], m0), d1 = cmul(M[1], m1), d2 = cmul(M[2], m2);
    const double dx = d0.x - d1.x + d2.x, dy = d0.y - d1.y + d2.y;
    psi = atan2(dy, dx) / (3.0 * M_PI);  // in units of pi
    double sp, cp;
    sincospi(psi, &sp, &cp);
    const double2 z = make_double2(cp / s, -sp / s);  // e^{-i pi psi} / s
    const double2 w00 = cmul(z, M[0]), w20 = cmul(z, M[6]);
    P[0] = make_double2(atan2(w00.y, w00.x) / M_PI, atan2(w20.y, w20.x) / M_PI);
    P[1] = cmul(z, M[1]);
    P[2] = cmul(z, M[2]);
    P[3] = cmul(z, M[3]);
}

// one thread per (target site, mu, l); LR = stored real type (fp64 input rounded to LR)
template <typename LR>
__global__ void convert_links_kernel(const LinkConvParams P) {
    using L2 = cplx_t<LR>;
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (gid >= P.vh * 16) return;
    const int64_t cb = gid >> 4;
    const int mu = (int)(gid >> 2) & 3;
    const int l = (int)gid & 3;
    int64_t r = cb;
    const int xh = (int)(r % P.lxh);
    r /= P.lxh;
    const int y = (int)(r % P.L[1]);
    r /= P.L[1];
    const int z = (int)(r % P.L[2]);
    const int t = (int)(r / P.L[2]);
    const int x = 2 * xh + ((P.parity + y + z + t) & 1);
    const bool is_long = l >= 2;
    const int back = (l == 1) ? 1 : (l == 3) ? 3 : 0;
    const double2* A = canon_link(P, is_long, mu, x, y, z, t, back);
    if (P.recon == 9 && is_long) {
        double2 M[9], Q[4];
        for (int i = 0; i < 3; ++i)
            for (int j = 0; j < 3; ++j) {
                double2 v = back ? A[3 * j + i] : A[3 * i + j];
                if (back) v.y = -v.y;
                M[3 * i + j] = v;
            }
        double psi;
        compress_9(M, P.s9, Q, psi);
        for (int e = 0; e < 4; ++e) static_cast<L2*>(P.links)[conv_index(P, mu, l, e, cb)] = to_cplx<L2>(Q[e]);
        if (P.paired)  // fp32 paired: entry 4 of the pair holds (psi_f, 0, psi_b, 0)
            static_cast<L2*>(P.links)[conv_index(P, mu, l, 4, cb)] = to_cplx<L2>(make_double2(psi, 0.0));
        else  // the psi pair: Nf's in .x, Nb's in .y
            reinterpret_cast<LR*>(static_cast<L2*>(P.links) + conv_index(P, mu, 2, kRecon9PhaseElem, cb))[l - 2] = (LR)psi;
        return;
    }
    const int rows = (P.recon == 12 && is_long) ? 2 : 3;
    for (int i = 0; i < rows; ++i)
        for (int j = 0; j < 3; ++j) {
            double2 v;
            if (back) {  // (A^dag)_{ij} = conj(A_{ji})
                v = A[3 * j + i];
                v.y = -v.y;
            } else {
                v = A[3 * i + j];
            }
            const int e = 3 * i + j;
            static_cast<L2*>(P.links)[conv_index(P, mu, l, e, cb)] = to_cplx<L2>(v);
        }
}

// fp64 internal layout S -> fp32 layout D (the mixed-precision solver's sloppy links, rounded
// once): same (mu, l, e) entries, D usually the paired fp32 layout of the same lane mapping; a
// recon-9 source is rebuilt and stored in full (D.recon = 18).
__global__ void convert_internal_kernel(const LinkConvParams S, const LinkConvParams D) {
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (gid >= S.vh * 16) return;
    const int64_t cb = gid >> 4;
    const int mu = (int)(gid >> 2) & 3;
    const int l = (int)gid & 3;
    if (S.recon == 9 && l >= 2) {  // recon-9 source: rebuilt in fp64, stored in full (D.recon 18)
        const double2* src = static_cast<const double2*>(S.links);
        double2 U[9];
        for (int e = 0; e < 4; ++e) U[e] = src[conv_index(S, mu, l, e, cb)];
        const double2 ph = src[conv_index(S, mu, 2, kRecon9PhaseElem, cb)];
        reconstruct_9(U, S.s9, l == 2 ? ph.x : ph.y);
        for (int e = 0; e < 9; ++e) static_cast<float2*>(D.links)[conv_index(D, mu, l, e, cb)] = to_cplx<float2>(U[e]);
        return;
    }
    const int stored = (S.recon == 12 && l >= 2) ? 6 : 9;
    for (int e = 0; e < stored; ++e)
        static_cast<float2*>(D.links)[conv_index(D, mu, l, e, cb)] =
            to_cplx<float2>(static_cast<const double2*>(S.links)[conv_index(S, mu, l, e, cb)]);
}

// Export (dslash_get_links): internal layout -> out[cb][mu][l][e] (double2), l = Ff, Fb, Nf, Nb.
// With recon-12 the long matrices' row 2 is not stored: exported as zeros.  With recon-9 the long
// matrices are exported reconstructed.
template <typename LR>
__global__ void export_links_kernel(const LinkConvParams P, double2* out) {
    using L2 = cplx_t<LR>;
    const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (gid >= P.vh * 16) return;
    const int64_t cb = gid >> 4;
    const int mu = (int)(gid >> 2) & 3;
    const int l = (int)gid & 3;
    const L2* links = static_cast<const L2*>(P.links);
    if (P.recon == 9 && l >= 2) {  // recon-9: exported reconstructed
        double2 U[9];
        for (int e = 0; e < 4; ++e) U[e] = widen(links[conv_index(P, mu, l, e, cb)]);
        double psi;
        if (P.paired) {
            psi = widen(links[conv_index(P, mu, l, 4, cb)]).x;
        } else {
            const double2 ph = widen(links[conv_index(P, mu, 2, kRecon9PhaseElem, cb)]);
            psi = l == 2 ? ph.x : ph.y;
        }
        reconstruct_9(U, P.s9, psi);
        for (int e = 0; e < 9; ++e) out[((cb * 4 + mu) * 4 + l) * 9 + e] = U[e];
        return;
    }
    const int stored = (P.recon == 12 && l >= 2) ? 6 : 9;
    for (int e = 0; e < 9; ++e) {
        double2 v = make_double2(0.0, 0.0);
        if (e < stored) v = widen(links[conv_index(P, mu, l, e, cb)]);
        out[((cb * 4 + mu) * 4 + l) * 9 + e] = v;
    }
}

// recon-12 admissibility: for every canonical long link N (fp64 input), the largest deviation
// |row2 - conj(row0 x row1)/s| over its 3 entries, as a non-negative double whose bit pattern
// orders like an unsigned integer (atomicMax on the bits).
__global__ void recon_check_kernel(const double2* lng, int64_t nmat, double inv_s, unsigned long long* max_bits) {
    const int64_t m = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    double err = 0.0;
    if (m < nmat) {
        const double2* A = lng + m * 9;
        double2 U[9];
        for (int e = 0; e < 9; ++e) U[e] = A[e];
        double2 R[9];
        for (int e = 0; e < 9; ++e) R[e] = U[e];
        reconstruct_row2(R, inv_s);
        for (int j = 0; j < 3; ++j) err = fmax(err, fmax(fabs(R[6 + j].x - U[6 + j].x), fabs(R[6 + j].y - U[6 + j].y)));
    }
    // warp max, then one atomic per warp
    for (int off = 16; off; off >>= 1) err = fmax(err, __shfl_xor_sync(0xffffffffu, err, off));
    if ((threadIdx.x & 31) == 0) atomicMax(max_bits, (unsigned long long)__double_as_longlong(err));
}

// recon-9 admissibility: for every canonical long link N (fp64 input) and its adjoint (the
// back-link form), the largest entry deviation of reconstruct_9(compress_9(M)) from M; atomicMax
// on the bits as in recon_check_kernel.  Fails where a link is not s e^{i psi} SU(3) with the
// handle's s, or lies too near the parameterisation's singular set (|a2|^2 + |a3|^2 -> 0).
__global__ void recon9_check_kernel(const double2* lng, int64_t nmat, double s, unsigned long long* max_bits) {
    const int64_t m = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    double err = 0.0;
    if (m < nmat) {
        const double2* A = lng + m * 9;
        for (int adj = 0; adj < 2; ++adj) {
            double2 M[9], U[9];
            for (int i = 0; i < 3; ++i)
                for (int j = 0; j < 3; ++j) {
                    double2 v = adj ? A[3 * j + i] : A[3 * i + j];
                    if (adj) v.y = -v.y;
                    M[3 * i + j] = v;
                }
            double psi;
            compress_9(M, s, U, psi);
            reconstruct_9(U, s, psi);
            for (int e = 0; e < 9; ++e) {
                const double dx = fabs(U[e].x - M[e].x), dy = fabs(U[e].y - M[e].y);
                err = (dx == dx && dy == dy) ? fmax(err, fmax(dx, dy)) : HUGE_VAL;  // NaN (singular): reject
            }
        }
    }
    for (int off = 16; off; off >>= 1) err = fmax(err, __shfl_xor_sync(0xffffffffu, err, off));
    if ((threadIdx.x & 31) == 0) atomicMax(max_bits, (unsigned long long)__double_as_longlong(err));
}

}  // namespace hisq
