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
// Mappings (chosen by measurement), one template dslash_kernel<LANES, ...>:
//   SITE (LANES 1): one thread per target site (the paper's 1LP decomposition, L59-87);
//   DIR2 (LANES 2): two lanes per site, two directions each, one __shfl_xor step;
//   DIR4 (LANES 4): four consecutive lanes per site, lane = mu, each lane streams that
//          direction's 4 matrices and the partial sums meet in two __shfl_xor steps (the
//          paper's 3LP-1 "site x direction + reduction" idea, L101-142, with shuffles instead
//          of local memory + barrier and without the row split, which replicates vector loads).
#pragma once

#include "common.cuh"

namespace hisq {

// Internal link layout, for a kernel with LANES lanes per site (lane j streams directions
// mu = k*LANES + j, k < 4/LANES).  Matrix l (0 = Ff (+1 hop), 1 = Fb (-1), 2 = Nf (+3),
// 3 = Nb (-3)) of direction mu at target site cb stores its elements e (row-major 3*i + j) at
//   links[(((base(l) + e) * K + k) * vh + cb) * LANES + j],   K = 4 / LANES,
// base(l) = 9 l without compression; with RECON = 12 the long matrices keep only rows 0 and 1
// (e < 6), base(2) = 18, base(3) = 24; with RECON = 9 they keep 4 entries (e < 4: (arg a1,
// arg c1), a2, a3, b1), base(2) = 18, base(3) = 22, and the pair (psi of Nf, psi of Nb) is
// element 26 (= base(2) + 8).  At every load instruction the lanes of a warp read one contiguous
// span, and consecutive elements of a matrix are 4*vh complex apart.
template <int RECON>
__host__ __device__ __forceinline__ int elem_base(int l) {
    return (RECON == 12 && l >= 2) ? 18 + (l - 2) * 6 : (RECON == 9 && l >= 2) ? 18 + (l - 2) * 4 : l * 9;
}
template <int RECON>
__host__ __device__ __forceinline__ int elems_of(int l) {
    return (RECON == 12 && l >= 2) ? 6 : (RECON == 9 && l >= 2) ? 4 : 9;
}
constexpr int kRecon9PhaseElem = 8;  // link_index<LANES, 9>(mu, 2, 8, ...) = the psi pair
template <int LANES, int RECON = 18>
__host__ __device__ __forceinline__ int64_t link_index(int mu, int l, int e, int64_t vh, int64_t cb) {
    constexpr int K = 4 / LANES;
    return ((((int64_t)(elem_base<RECON>(l) + e) * K + mu / LANES) * vh + cb) * LANES) + (mu % LANES);
}

// fp32 links ("paired" layout): entry e of the forward and the backward matrix of one kind
// (Ff, Fb: pair j = 0; Nf, Nb: j = 1) share one 16-byte float4, so every lane issues 16-byte
// loads as in fp64 (no padding: a matrix pair is 2 x 72 B):
//   links4[(((pbase(j) + e) * K + k) * vh + cb) * LANES + lane],  pbase(0) = 0, pbase(1) = 9.
template <int LANES>
__host__ __device__ __forceinline__ int64_t link_index_paired(int mu, int j, int e, int64_t vh, int64_t cb) {
    constexpr int K = 4 / LANES;
    return ((((int64_t)(j * 9 + e) * K + mu / LANES) * vh + cb) * LANES) + (mu % LANES);
}

// Row 2 of s*W, W in SU(3), from rows 0 and 1: conj(r0 x r1) / s  (QUDA/MILC "recon-12";
// the back-link N(x-3mu)^dag = s W^dag has the same form).  inv_s = 1/s.
template <typename V2, typename R>
__device__ __forceinline__ void reconstruct_row2(V2 U[9], R inv_s) {
#pragma unroll
    for (int j = 0; j < 3; ++j) {
        const int j1 = (j + 1) % 3, j2 = (j + 2) % 3;
        // x = r0[j1] r1[j2] - r0[j2] r1[j1]
        R xr = U[j1].x * U[3 + j2].x - U[j1].y * U[3 + j2].y;
        R xi = U[j1].x * U[3 + j2].y + U[j1].y * U[3 + j2].x;
        xr -= U[j2].x * U[3 + j1].x - U[j2].y * U[3 + j1].y;
        xi -= U[j2].x * U[3 + j1].y + U[j2].y * U[3 + j1].x;
        U[6 + j].x = xr * inv_s;
        U[6 + j].y = -xi * inv_s;
    }
}

// recon-9 (QUDA's 8 SU(3) parameters + one phase for the long links with folded staggered
// phases): M = s e^{i psi} W with W in SU(3), s > 0 one real scale per handle, psi = arg(det M)/3.
// Stored: U[0] = (arg a1, arg c1) / pi, U[1] = a2, U[2] = a3, U[3] = b1, with rows a, b, c of W,
// and psi / pi (in the direction's psi pair).
// Unitarity and det W = 1 give |a1|^2 = 1 - |a2|^2 - |a3|^2, |c1|^2 = |a2|^2 + |a3|^2 - |b1|^2, and
// (rows orthogonal to a, b = conj(c x a), c = conj(a x b)), with n = |a2|^2 + |a3|^2:
//   b2 = -(a1* b1 a2 + a3* c1*) / n,   b3 = (a2* c1* - a1* b1 a3) / n,
//   c2 = (a3* b1* - a1* c1 a2) / n,    c3 = -(a2* b1* + a1* c1 a3) / n.
template <typename V2>
__device__ __forceinline__ V2 cmul(V2 a, V2 b) {
    return V2{a.x * b.x - a.y * b.y, a.x * b.y + a.y * b.x};
}
template <typename V2>
__device__ __forceinline__ V2 cconj(V2 a) {
    return V2{a.x, -a.y};
}
// fp32 reconstruction (recon-9 is rebuilt in the precision its parameters are stored in).  FAST
// (the default): the hardware approximations, MUFU sin/cos of pi*a for |a| <= 1 (abs. error ~4e-7)
// and rsqrt; otherwise the accurate fp32 routines (sincospif, sqrtf).  Measured at 32^4
// (profiles/r02/recon9_accuracy/): both give the same normwise error, 2.0e-6 for f32 and mixed
// recon-9 (recon-18: 2.9e-7 / 2.8e-8), because the error comes from rounding the STORED parameters
// to fp32 and the parameterisation's conditioning (|c1| = sqrt(n - |b1|^2) cancels, and b2..c3
// divide by n = |a2|^2 + |a3|^2), not from the rebuild arithmetic; the accurate routines only cost
// time (mixed 83.0 -> 91.9 us).  fp64 keeps the libdevice routines.
template <bool FAST>
__device__ __forceinline__ void sincospi_r(double a, double* s, double* c) { sincospi(a, s, c); }
template <bool FAST>
__device__ __forceinline__ void sincospi_r(float a, float* s, float* c) {
    if (FAST)
        __sincosf(a * 3.14159265358979f, s, c);
    else
        sincospif(a, s, c);
}
template <bool FAST>
__device__ __forceinline__ double sqrt0_r(double x) { return sqrt(fmax(x, 0.0)); }
template <bool FAST>
__device__ __forceinline__ float sqrt0_r(float x) { return FAST ? (x > 0.f ? x * rsqrtf(x) : 0.f) : sqrtf(fmaxf(x, 0.f)); }
__device__ __forceinline__ double rcp_r(double x) { return 1.0 / x; }
__device__ __forceinline__ float rcp_r(float x) { return __frcp_rn(x); }

// HISQ_RECON9_FAST (compile-time, default 1): the hardware approximations in the fp32 rebuild
#ifndef HISQ_RECON9_FAST
#define HISQ_RECON9_FAST 1
#endif

// SCALE = false leaves U = W and only returns z = s e^{i pi psi} (the stencil multiplies the
// 3-vector W v by z instead of the 9 entries of W)
template <bool SCALE = true, bool FAST = false, typename V2, typename R>
__device__ __forceinline__ V2 reconstruct_9(V2 U[9], R s, R psi) {
    const V2 a2 = U[1], a3 = U[2], b1 = U[3];
    const R n = a2.x * a2.x + a2.y * a2.y + a3.x * a3.x + a3.y * a3.y;
    const R a1m = sqrt0_r<FAST>(R(1) - n);
    const R c1m = sqrt0_r<FAST>(n - (b1.x * b1.x + b1.y * b1.y));
    R sa, ca, sc, cc, sp, cp;
    sincospi_r<FAST>(U[0].x, &sa, &ca);  // angles are stored in units of pi: no large-argument reduction
    sincospi_r<FAST>(U[0].y, &sc, &cc);
    sincospi_r<FAST>(psi, &sp, &cp);
    const V2 a1{a1m * ca, a1m * sa}, c1{c1m * cc, c1m * sc};
    const R inv = rcp_r(n);
    const V2 a1b1 = cmul(cconj(a1), b1), a1c1 = cmul(cconj(a1), c1);
    const V2 t0 = cmul(a1b1, a2), t1 = cmul(cconj(a3), cconj(c1));
    const V2 t2 = cmul(cconj(a2), cconj(c1)), t3 = cmul(a1b1, a3);
    const V2 t4 = cmul(cconj(a3), cconj(b1)), t5 = cmul(a1c1, a2);
    const V2 t6 = cmul(cconj(a2), cconj(b1)), t7 = cmul(a1c1, a3);
    const V2 b2{-(t0.x + t1.x) * inv, -(t0.y + t1.y) * inv};
    const V2 b3{(t2.x - t3.x) * inv, (t2.y - t3.y) * inv};
    const V2 c2{(t4.x - t5.x) * inv, (t4.y - t5.y) * inv};
    const V2 c3{-(t6.x + t7.x) * inv, -(t6.y + t7.y) * inv};
    const V2 z{s * cp, s * sp};
    if (SCALE) {
        U[0] = cmul(z, a1);
        U[1] = cmul(z, a2);
        U[2] = cmul(z, a3);
        U[3] = cmul(z, b1);
        U[4] = cmul(z, b2);
        U[5] = cmul(z, b3);
        U[6] = cmul(z, c1);
        U[7] = cmul(z, c2);
        U[8] = cmul(z, c3);
    } else {
        U[0] = a1;
        U[4] = b2;
        U[5] = b3;
        U[6] = c1;
        U[7] = c2;
        U[8] = c3;
    }
    return z;
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

// sites per block of the site-blocked multi-RHS vector layout (dslash_apply_multi_blocked)
constexpr int kVBlk = 16;

template <typename V2>
struct SrcRef {
    const V2* p;  // colour component c at p[c * stride]
    int64_t stride;
    bool ghost;   // the source lies in a ghost face (GHOST kernels only)
};

// Address of psi(x + h mu^).  GHOST: directions in P.halo_mask read the depth-3 ghost faces
// outside [0, L); otherwise coordinates wrap periodically (two conditional steps suffice for
// |h| <= 3 and L >= 2).
template <typename V2, bool GHOST, bool VBLK = false>
__device__ __forceinline__ SrcRef<V2> source(const StencilParams& P, const void* in, int mu, int h, const Site& s,
                                             int rhs) {
    const int c = mu == 0 ? s.x : mu == 1 ? s.y : mu == 2 ? s.z : s.t;
    const int L = P.L[mu];
    const int cn = c + h;
    int cw = cn;
    if (cw < 0) cw += L;
    if (cw < 0) cw += L;
    if (cw >= L) cw -= L;
    if (cw >= L) cw -= L;
    int64_t idx;
    int64_t st = 1;
    if (mu == 0) {
        idx = s.cb - s.xh + (cw >> 1);
    } else {
        st = mu == 1 ? (int64_t)P.lxh : mu == 2 ? (int64_t)P.lxh * P.L[1] : (int64_t)P.lxh * P.L[1] * P.L[2];
        idx = s.cb + (int64_t)(cw - c) * st;
    }
    // site-blocked vectors (dslash_apply_multi_blocked): (rhs, colour c) of site idx at
    // [idx / 16][rhs * 3 + c][idx % 16], P.vblk complex per 16-site block; the ghost faces are
    // blocked the same way over their face index
    const V2* local = VBLK ? static_cast<const V2*>(in) + (idx >> 4) * P.vblk + (idx & 15) + rhs * 3 * kVBlk
                           : static_cast<const V2*>(in) + (int64_t)rhs * 3 * P.vh + idx;
    const int64_t lstride = VBLK ? (int64_t)kVBlk : P.vh;
    if (!GHOST || mu < 2) return {local, lstride, false};
    // branch-free choice between the local site and the ghost face: the lanes of a site walk
    // different directions, so a branch here would diverge within the warp
    const bool ghost = ((P.halo_mask >> mu) & 1) && (cn < 0 || cn >= L);
    const int side = cn >= L;
    // face index f of depth d = (side ? cn - L : cn + 3): t face [d][z][y][xh] = cb + st (d - t),
    // z face [t][d][y][xh] = cb + st (d - z) + st (3 - Lz) t (st = the direction's cb stride)
    const int64_t f = s.cb + st * (h + (side ? -L : 3)) + (mu == 2 ? st * (3 - P.L[2]) * (int64_t)s.t : 0);
    const int64_t fv = P.face_vh[mu];
    const V2* gp = VBLK ? static_cast<const V2*>(P.ghost[mu][side]) + (f >> 4) * P.vblk + (f & 15) + rhs * 3 * kVBlk
                        : static_cast<const V2*>(P.ghost[mu][side]) + (int64_t)rhs * 3 * fv + f;
    // local pass of the split-by-direction overlap: the face is still in flight, so a ghost hop
    // reads the (valid) wrapped local address and the caller zeroes the vector
    const bool use_face = ghost && P.halo_pass != kPassLocal;
    return {use_face ? gp : local, use_face ? (VBLK ? (int64_t)kVBlk : fv) : lstride, ghost};
}

// ---------------------------------------------------------------- staged neighbour tile
// DSLASH_OPT_STAGE (the 3LP-1 kernel's local-memory staging):
// a block owns one tile = TY full x-rows y0 .. y0+TY-1 at one (z, t).  Its 8 x- and y-hops per
// site read source rows y0-3 .. y0+TY+2 of that (z, t) plane, which the TMA engine copies into
// shared memory once per tile (cp.async.bulk, one copy per contiguous run of rows and
// (rhs, colour)), instead of 8 gathers per site from L1/L2.  z and t hops, whose sources no
// other site of the tile reads, stay global loads.  x and y are never partitioned, so every
// staged row is local.  Layout: sv[((r * 3 + c) * rows + i) * lxh + xh], row i <-> y = y0-3+i.
template <typename V2>
struct StageTile {
    V2* sv;          // shared-memory tile
    uint64_t* bar;   // mbarrier: the tile's bulk copies complete on it (phase 0)
    int y0;          // first row of the tile
    int rows;        // TY + 6
    int64_t plane0;  // cb offset of (xh = 0, y = 0) in the tile's (z, t) plane
    uint32_t sbase;  // shared-state-space address of sv
};

// thread 0: one bulk copy per (rhs, colour) and contiguous run of rows (the y wrap splits it)
template <typename V2>
__device__ __forceinline__ void stage_tile_issue(const StencilParams& P, const void* in, const StageTile<V2>& T, int nr,
                                                 uint64_t pol) {
    const int Ly = P.L[1], lxh = P.lxh, rows = T.rows;
    const uint32_t row_bytes = (uint32_t)(lxh * sizeof(V2));
    mbar_arrive_expect_tx(T.bar, (uint32_t)(nr * 3 * rows) * row_bytes);
    const V2* src = static_cast<const V2*>(in);
    for (int i = 0; i < rows;) {
        int y = (T.y0 - 3 + i) % Ly;
        if (y < 0) y += Ly;
        const int n = min(rows - i, Ly - y);
        for (int rc = 0; rc < nr * 3; ++rc)
            bulk_g2s(T.sv + ((int64_t)rc * rows + i) * lxh, src + (int64_t)rc * P.vh + T.plane0 + (int64_t)y * lxh,
                     (uint32_t)n * row_bytes, T.bar, pol);
        i += n;
    }
}

// shared address of psi(x + h mu^), colour 0, right-hand side `rhs`, for mu = 0 (x) or 1 (y);
// colour c / rhs r lie c (3 r) planes of rows * lxh complex further
template <typename V2>
__device__ __forceinline__ uint32_t staged_addr(const StencilParams& P, const StageTile<V2>& T, uint32_t sbase, int mu,
                                                int h, const Site& s, int rhs) {
    const int L = P.L[0];
    int cw = s.x + h;
    if (cw < 0) cw += L;
    if (cw < 0) cw += L;
    if (cw >= L) cw -= L;
    if (cw >= L) cw -= L;
    const bool ymove = mu != 0;
    const int row = s.y - T.y0 + 3 + (ymove ? h : 0);
    const int xh = ymove ? s.xh : (cw >> 1);
    return sbase + (uint32_t)((rhs * 3 * T.rows + row) * P.lxh + xh) * (uint32_t)sizeof(V2);
}

// Wait for the tile's bulk copies; the returned base address comes out of the waiting asm, so no
// shared load addressed from it can be scheduled above the wait (the loads below need not be
// volatile and can be batched freely).
__device__ __forceinline__ uint32_t stage_wait(uint64_t* bar, uint32_t sbase) {
    uint32_t b;
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "SWAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\t"
        "@!p bra SWAIT_%=;\n\t"
        "mov.b32 %0, %2;\n}"
        : "=r"(b)
        : "r"(smem_addr(bar)), "r"(sbase)
        : "memory");
    return b;
}

__device__ __forceinline__ double2 lds_at(uint32_t a, double2*) {
    double2 r;
    asm("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(r.x), "=d"(r.y) : "r"(a));
    return r;
}
__device__ __forceinline__ float2 lds_at(uint32_t a, float2*) {
    float2 r;
    asm("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(r.x), "=f"(r.y) : "r"(a));
    return r;
}

// one neighbour colour component: from the staged tile (shared address sa + off_b) or from global
template <typename V2>
__device__ __forceinline__ V2 ld_src(bool staged, uint32_t sa, uint32_t off_b, const V2* p, uint64_t pol,
                                     bool no_l1 = false) {
    return staged ? lds_at(sa + off_b, (V2*)nullptr) : no_l1 ? ld_reuse_na(p, pol) : ld_reuse(p, pol);
}

// v = 0 when z (a select, so acc + U * 0 leaves acc's value unchanged without a branch)
template <typename V2>
__device__ __forceinline__ void zero_if(V2& v, bool z) {
    v.x = z ? decltype(v.x)(0) : v.x;
    v.y = z ? decltype(v.y)(0) : v.y;
}

// acc (+/-)= U v for a 3x3 matrix whose 9 elements are U[e]
template <bool SUB, typename V2>
__device__ __forceinline__ void matvec_acc(V2 acc[3], const V2 U[9], const V2 v[3]) {
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

// z / t hop vectors bypass L1: their other consumers (targets in neighbouring z / t planes) run in
// other blocks, normally on other SMs, so their lines only evicted the x / y rows this block
// reuses.  Measured A/B (profiles/r02/mrhs/ab_zt_no_l1.txt): 8 RHS L1 hit rate 21% -> 31%, time
// +0.5% better; 1 RHS unchanged (179.96 us either way).
#ifndef HISQ_ZT_NO_L1
#define HISQ_ZT_NO_L1 1
#endif
constexpr bool kZtNoL1 = HISQ_ZT_NO_L1 != 0;

// ---------------------------------------------------------------- the stencil kernel
// LANES consecutive threads per target site (1 = thread per site, the paper's 1LP mapping;
// 4 = one lane per direction, the paper's 3LP-1 site x direction split with a shuffle
// reduction instead of local memory + barrier).  MINB = minimum resident 256-thread blocks per
// SM, which caps registers (2 -> 128, 3 -> 80, 4 -> 64) and so trades per-thread ILP against
// occupancy.  NRHS right-hand sides ([NRHS][3][vh] vectors) are register-blocked: each thread
// loads a link matrix once and applies it to NRHS vectors, so the link stream is shared
// (the L25 Domain-Wall intensity argument).  GHOST selects the boundary
// variant that reads halo faces.  LR is the real type of the stored links, VR that of the
// vectors and of the accumulation (double/double = fp64, float/float = fp32, float/double =
// mixed: fp32 links widened to fp64 before the FMAs).  RECON 12 rebuilds row 2 of the long
// links.  The summation order per (site, rhs) is the same for every NRHS, MINB and block size.
// The per-thread body: thread gid of the box enumeration (LANES consecutive gids per site).  All
// LANES threads of a site must call it together (shuffle reduction).
// RHSL > 1: the site's right-hand sides are split over RHSL adjacent thread groups, each
// register-blocking NRHS of them (rhs = rl * NRHS + r); the groups of a site issue identical link
// addresses in one warp instruction, so each sector is fetched once.
// STAGED: x/y neighbours come from the block's shared-memory tile T (dslash_stage_kernel).  The
// staged kernel visits the global (z, t) directions first and the tile's (x, y) ones last, so
// the tile's bulk copies land while the z/t links and neighbours stream (a different summation
// order from the unstaged kernel: equal within the fp64 tolerance, not bitwise).
template <typename LR, typename VR, int LANES, bool GHOST, int RECON, int NRHS, int RHSL = 1, bool STAGED = false,
          bool VBLK = false>
__device__ __forceinline__ void dslash_body(const StencilParams& P, const int64_t gid, const int64_t site_end,
                                            const StageTile<cplx_t<VR>> T = {}) {
    static_assert(LANES == 1 || LANES == 2 || LANES == 4, "LANES must divide 4");
    static_assert(!STAGED || LANES <= 2, "the staged tile serves LANES 1 and 2");
    using L2 = cplx_t<LR>;
    using V2 = cplx_t<VR>;
    constexpr int K = 4 / LANES;
    constexpr int kFirstStaged = LANES == 1 ? 2 : 1;  // first loop step that reads the tile
    const int lane = (LANES == 1) ? 0 : (int)(gid & (LANES - 1));
    // thread -> (site, right-hand-side group).  LANES 1 x RHSL 2 in a one-dimensional grid of
    // whole warps (not the staged kernel): each quarter-warp (8 lanes) takes 8 consecutive sites of
    // ONE group, so a 16-byte load of a quarter-warp touches one 128-byte line (one L1 wavefront)
    // instead of two; the warp still covers the same 16 sites
    constexpr bool kQuarterRuns = LANES == 1 && (RHSL == 2 || RHSL == 4) && !STAGED;
    const int rl = (RHSL == 1)    ? 0
                   : kQuarterRuns ? (int)((gid >> 3) % RHSL)
                                  : (int)((gid / LANES) % RHSL);
    const int64_t site = kQuarterRuns ? (gid >> 5) * (32 / RHSL) + ((gid >> 3) / RHSL) % (4 / RHSL) * 8 + (gid & 7)
                                      : gid / (LANES * RHSL);
    const bool valid = site < site_end;
    if (LANES == 1 && !valid) return;
    V2 acc[NRHS][3];
#pragma unroll
    for (int r = 0; r < NRHS; ++r)
#pragma unroll
        for (int c = 0; c < 3; ++c) acc[r][c].x = acc[r][c].y = VR(0);
    Site s;
    if (valid) {
        const uint64_t pol_stream = policy_evict_first();
        const uint64_t pol_keep = policy_evict_last();
        s = decode_site(P, site);
        const L2* links = static_cast<const L2*>(P.links);
        // Programmatic dependent launch (DSLASH_OPT_PDL): the links are read-only, so the first
        // matrix (unpaired layouts) is fetched before waiting for the previous grid; psi (and the
        // ghosts) are read, and chi written, only after griddepcontrol.wait, whose asm yields the
        // psi base pointer so no psi load can be hoisted above it.  Without a PDL launch the wait
        // returns at once.
        // (staged: thread 0 issues the tile's bulk copies right after the wait, before any link is
        // in flight, so the issue loop's registers never coexist with a held matrix)
        const void* in = nullptr;
        if constexpr (STAGED) {
            asm volatile("griddepcontrol.wait;\n\tmov.b64 %0, %1;" : "=l"(in) : "l"(P.in) : "memory");
            if (threadIdx.x == 0) stage_tile_issue(P, in, T, NRHS * RHSL, pol_keep);
        }
        V2 U0[9];
        // (not in the ghost pass, whose first hop is never a ghost hop for LANES 1 / 2)
        if (sizeof(LR) != 4 && !(GHOST && P.halo_pass == kPassGhost)) {
            const L2* lp0 = links + link_index<LANES, RECON>((STAGED ? K - 1 : 0) * LANES + lane, 0, 0, P.vh, s.cb);
#pragma unroll
            for (int e = 0; e < 9; ++e) U0[e] = to_cplx<V2>(widen(ld_stream(lp0 + (int64_t)e * 4 * P.vh, pol_stream)));
        }
        if constexpr (!STAGED) asm volatile("griddepcontrol.wait;\n\tmov.b64 %0, %1;" : "=l"(in) : "l"(P.in) : "memory");
        const uint32_t plane_b = STAGED ? (uint32_t)(T.rows * P.lxh * sizeof(V2)) : 0u;  // bytes per staged plane
        uint32_t sbase = 0;  // the tile's shared address, valid once stage_wait returned it
#pragma unroll
        for (int kk = 0; kk < K; ++kk) {
            const int k = STAGED ? K - 1 - kk : kk;
            const int mu = k * LANES + lane;
            // compile-time after unrolling: LANES 1 -> mu = k; LANES 2 -> k == 0 is (x, y)
            const bool stg = STAGED && (LANES == 1 ? k < 2 : k == 0);
            if constexpr (STAGED) {
                if (kk == kFirstStaged) sbase = stage_wait(T.bar, T.sbase);
            }
            if constexpr (sizeof(LR) == 4) {
                // fp32 links, paired layout: one 16-byte load feeds the forward and the backward
                // matrix of a kind; the FMA order is that of the unpaired loop (l = 0, 1, 2, 3)
                const float4* links4 = static_cast<const float4*>(P.links);
                float4 L9w[5];  // recon-9: the long pair's entries, fetched with the fat pair (latency)
                if constexpr (RECON == 9) {
                    const float4* lq = links4 + link_index_paired<LANES>(mu, 1, 0, P.vh, s.cb);
#pragma unroll
                    for (int e = 0; e < 5; ++e) L9w[e] = ld_stream(lq + (int64_t)e * 4 * P.vh, pol_stream);
                }
#pragma unroll
                for (int j = 0; j < 2; ++j) {
                    const int hop = j ? 3 : 1;
                    if (GHOST && P.halo_pass == kPassGhost) {
                        // ghost pass of the split-by-direction overlap: skip a kind neither of
                        // whose two hops reaches a ghost face (no link bytes either)
                        const bool ga = source<V2, GHOST>(P, in, mu, hop, s, 0).ghost;
                        const bool gb = source<V2, GHOST>(P, in, mu, -hop, s, 0).ghost;
                        if (!(ga || gb)) continue;
                    }
                    const float4* lp = links4 + link_index_paired<LANES>(mu, j, 0, P.vh, s.cb);
                    V2 Ua[9], Ub[9];
#pragma unroll
                    for (int e = 0; e < elems_of<RECON>(2 * j); ++e) {
                        const float4 w = (RECON == 9 && j == 1) ? L9w[e] : ld_stream(lp + (int64_t)e * 4 * P.vh, pol_stream);
                        Ua[e] = to_cplx<V2>(widen(make_float2(w.x, w.y)));
                        Ub[e] = to_cplx<V2>(widen(make_float2(w.z, w.w)));
                    }
                    if (elems_of<RECON>(2 * j) == 6) {
                        reconstruct_row2(Ua, (VR)P.long_inv_scale);
                        reconstruct_row2(Ub, (VR)P.long_inv_scale);
                    }
                    V2 za, zb;  // recon-9: Nf = za Wa, Nb = zb Wb (the psi pair is entry 4: (psi_f, 0, psi_b, 0))
                    if constexpr (RECON == 9) {
                        if (j == 1) {
                            // rebuilt in fp32, the precision the parameters are stored in (mixed
                            // widens the result; its accuracy is set by the fp32 parameters, see
                            // sincospi_r)
                            float2 fa[9], fb[9];
#pragma unroll
                            for (int e = 0; e < 4; ++e) {
                                fa[e] = make_float2(L9w[e].x, L9w[e].y);
                                fb[e] = make_float2(L9w[e].z, L9w[e].w);
                            }
                            const float2 zfa = reconstruct_9<false, HISQ_RECON9_FAST>(fa, (float)P.long_scale, L9w[4].x);
                            const float2 zfb = reconstruct_9<false, HISQ_RECON9_FAST>(fb, (float)P.long_scale, L9w[4].z);
#pragma unroll
                            for (int e = 0; e < 9; ++e) {
                                Ua[e] = to_cplx<V2>(widen(fa[e]));
                                Ub[e] = to_cplx<V2>(widen(fb[e]));
                            }
                            za = to_cplx<V2>(widen(zfa));
                            zb = to_cplx<V2>(widen(zfb));
                        }
                    }
#pragma unroll
                    for (int sub = 0; sub < 2; ++sub) {
                        const SrcRef<V2> src = stg ? SrcRef<V2>{nullptr, 0, false}
                                                   : source<V2, GHOST, VBLK>(P, in, mu, sub ? -hop : hop, s, rl * NRHS);
                        const uint32_t sa = stg ? staged_addr<V2>(P, T, sbase, mu, sub ? -hop : hop, s, rl * NRHS) : 0u;
                        if (GHOST && P.halo_pass == kPassGhost && !src.ghost) continue;
                        const bool zap = GHOST && P.halo_pass == kPassLocal && src.ghost;
#pragma unroll
                        for (int r = 0; r < NRHS; ++r) {
                            const int64_t roff = (int64_t)r * 3 * src.stride;
                            V2 v[3];
#pragma unroll
                            for (int c = 0; c < 3; ++c) {
                                v[c] = ld_src(stg, sa, (uint32_t)(r * 3 + c) * plane_b, src.p + roff + c * src.stride,
                                              pol_keep, kZtNoL1 && mu >= 2);
                                if (GHOST) zero_if(v[c], zap);
                            }
                            if (RECON == 9 && j == 1) {
                                V2 w3[3];
#pragma unroll
                                for (int i = 0; i < 3; ++i) w3[i].x = w3[i].y = VR(0);
                                matvec_acc<false>(w3, sub ? Ub : Ua, v);
#pragma unroll
                                for (int i = 0; i < 3; ++i) {
                                    if (sub)
                                        cmsub(acc[r][i], zb, w3[i]);
                                    else
                                        cmadd(acc[r][i], za, w3[i]);
                                }
                            } else if (sub) {
                                matvec_acc<true>(acc[r], Ub, v);
                            } else {
                                matvec_acc<false>(acc[r], Ua, v);
                            }
                        }
                    }
                }
            } else {
            V2 ph9;       // recon-9: (psi of Nf, psi of Nb) of direction mu
            V2 L9[2][4];  // recon-9: the stored parameters of Nf, Nb
#pragma unroll
            for (int l = 0; l < 4; ++l) {
                const int h = (l == 0) ? 1 : (l == 1) ? -1 : (l == 2) ? 3 : -3;
                if constexpr (RECON == 9) {
                    // the direction's long-link parameters are fetched with its first (fat) matrix,
                    // so their latency overlaps the fat matvecs rather than the reconstruction
                    if (l == 0) {
                        ph9 = to_cplx<V2>(widen(
                            ld_stream(links + link_index<LANES, 9>(mu, 2, kRecon9PhaseElem, P.vh, s.cb), pol_stream)));
#pragma unroll
                        for (int q = 0; q < 2; ++q)
#pragma unroll
                            for (int e = 0; e < 4; ++e)
                                L9[q][e] = to_cplx<V2>(widen(ld_stream(
                                    links + link_index<LANES, 9>(mu, 2 + q, 0, P.vh, s.cb) + (int64_t)e * 4 * P.vh,
                                    pol_stream)));
                    }
                }
                const SrcRef<V2> src = stg ? SrcRef<V2>{nullptr, 0, false} : source<V2, GHOST, VBLK>(P, in, mu, h, s, rl * NRHS);
                const uint32_t sa = stg ? staged_addr<V2>(P, T, sbase, mu, h, s, rl * NRHS) : 0u;
                // split-by-direction passes: the ghost pass takes only the ghost hops (the link of
                // a skipped hop is not read); the local pass stays branch-free, so loads can be
                // hoisted as in the unsplit kernel: a ghost hop multiplies a zeroed vector (its
                // link is read in both passes, 144 B per ghost hop)
                if (GHOST && P.halo_pass == kPassGhost && !src.ghost) continue;
                const bool zap = GHOST && P.halo_pass == kPassLocal && src.ghost;
                const L2* lp = links + link_index<LANES, RECON>(mu, l, 0, P.vh, s.cb);
                V2 U[9];
                if (kk == 0 && l == 0 && !(GHOST && P.halo_pass == kPassGhost)) {
#pragma unroll
                    for (int e = 0; e < 9; ++e) U[e] = U0[e];
                } else if (RECON == 9 && l >= 2) {
#pragma unroll
                    for (int e = 0; e < 4; ++e) U[e] = L9[l - 2][e];
                } else {
#pragma unroll
                    for (int e = 0; e < elems_of<RECON>(l); ++e)
                        U[e] = to_cplx<V2>(widen(ld_stream(lp + (int64_t)e * 4 * P.vh, pol_stream)));
                }
                if (elems_of<RECON>(l) == 6) reconstruct_row2(U, (VR)P.long_inv_scale);
                V2 z9;  // recon-9: N = z9 W
                if constexpr (RECON == 9) {
                    if (l >= 2) z9 = reconstruct_9<false>(U, (VR)P.long_scale, l == 2 ? ph9.x : ph9.y);
                }
#pragma unroll
                for (int r = 0; r < NRHS; ++r) {
                    const int64_t roff = (int64_t)r * 3 * src.stride;  // [rhs][3][vh or face_vh]
                    V2 v[3];
#pragma unroll
                    for (int c = 0; c < 3; ++c) {
                        v[c] = ld_src(stg, sa, (uint32_t)(r * 3 + c) * plane_b, src.p + roff + c * src.stride, pol_keep,
                                      kZtNoL1 && mu >= 2);
                        if (GHOST) zero_if(v[c], zap);
                    }
                    if (RECON == 9 && l >= 2) {
                        V2 w[3];
#pragma unroll
                        for (int i = 0; i < 3; ++i) w[i].x = w[i].y = VR(0);
                        matvec_acc<false>(w, U, v);
#pragma unroll
                        for (int i = 0; i < 3; ++i) {
                            if (l & 1)
                                cmsub(acc[r][i], z9, w[i]);
                            else
                                cmadd(acc[r][i], z9, w[i]);
                        }
                    } else if (l & 1) {
                        matvec_acc<true>(acc[r], U, v);
                    } else {
                        matvec_acc<false>(acc[r], U, v);
                    }
                }
            }
            }  // unpaired links
        }
    }
    if (LANES > 1) {
        // butterfly over the lanes of a site: every lane ends with the same bits
        // (((p0+p1)+(p2+p3)) by commutativity of each pairwise add)
#pragma unroll
        for (int r = 0; r < NRHS; ++r)
#pragma unroll
            for (int c = 0; c < 3; ++c) {
#pragma unroll
                for (int off = 1; off < LANES; off <<= 1) {
                    acc[r][c].x += __shfl_xor_sync(0xffffffffu, acc[r][c].x, off);
                    acc[r][c].y += __shfl_xor_sync(0xffffffffu, acc[r][c].y, off);
                }
            }
    }
    if (!valid) return;
    if (GHOST && P.halo_pass == kPassGhost) {
        // ghost pass: chi = (local pass's partial sum) + (ghost hops), read back per colour this
        // lane stores below
#pragma unroll
        for (int r = 0; r < NRHS; ++r) {
            const V2* prev = static_cast<const V2*>(P.out) + (int64_t)(rl * NRHS + r) * 3 * P.vh + s.cb;
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                const bool mine = LANES == 1 || (LANES == 2 ? (lane == 0) == (c < 2) : lane == c);
                if (mine) {
                    const V2 o = prev[c * P.vh];
                    acc[r][c].x = o.x + acc[r][c].x;
                    acc[r][c].y = o.y + acc[r][c].y;
                }
            }
        }
    }
#pragma unroll
    for (int r = 0; r < NRHS; ++r) {
        // colour c of this (site, rhs) at out[c * cs]: planar [rhs][3][vh], or site-blocked
        V2* out = VBLK ? static_cast<V2*>(P.out) + (s.cb >> 4) * P.vblk + (s.cb & 15) + (rl * NRHS + r) * 3 * kVBlk
                       : static_cast<V2*>(P.out) + (int64_t)(rl * NRHS + r) * 3 * P.vh + s.cb;
        const int64_t cs = VBLK ? kVBlk : P.vh;
        if (LANES == 1) {
#pragma unroll
            for (int c = 0; c < 3; ++c) st_stream(out + c * cs, acc[r][c]);
        } else if (LANES == 2) {
            if (lane == 0) {
                st_stream(out, acc[r][0]);
                st_stream(out + cs, acc[r][1]);
            } else {
                st_stream(out + 2 * cs, acc[r][2]);
            }
        } else {
            if (lane < 3) st_stream(out + lane * cs, lane == 0 ? acc[r][0] : lane == 1 ? acc[r][1] : acc[r][2]);
        }
    }
    if constexpr (GHOST) {
        // producer push (DSLASH_OPT_PUSH): a site in the 3 bottom (top) slices of a pushed
        // direction is a source of the minus (plus) neighbour's next apply; store its output
        // straight into that neighbour's ghost face (peer memory), in the face order
        // halo_start's copies use, so the next apply exchanges no bytes.  The local pass of the
        // split by direction holds partial sums only and never pushes.
        if (P.push_mask && P.halo_pass != kPassLocal) {
#pragma unroll
            for (int mu = 2; mu < 4; ++mu) {
                if (!((P.push_mask >> mu) & 1)) continue;
                const int c = mu == 2 ? s.z : s.t;
                const int L = P.L[mu];
                const int64_t fv = P.face_vh[mu];
#pragma unroll
                for (int side = 0; side < 2; ++side) {
                    // (with L = 4 a slice can be both a bottom and a top slice)
                    if (side == 0 ? c >= 3 : c < L - 3) continue;
                    const int d = side ? c - (L - 3) : c;
                    const int64_t f = (mu == 3)
                                          ? s.xh + (int64_t)P.lxh * (s.y + (int64_t)P.L[1] * (s.z + (int64_t)P.L[2] * d))
                                          : s.xh + (int64_t)P.lxh * (s.y + (int64_t)P.L[1] * (d + 3 * (int64_t)s.t));
#pragma unroll
                    for (int r = 0; r < NRHS; ++r) {
                        V2* g = static_cast<V2*>(P.push[mu][side]) + (int64_t)(rl * NRHS + r) * 3 * fv + f;
#pragma unroll
                        for (int cc = 0; cc < 3; ++cc) {
                            const bool mine = LANES == 1 || (LANES == 2 ? (lane == 0) == (cc < 2) : lane == cc);
                            if (mine) g[cc * fv] = acc[r][cc];
                        }
                    }
                }
            }
        }
    }
}

// VBLK: the source and output vectors are in the site-blocked layout (dslash_apply_multi_blocked)
template <typename LR, typename VR, int LANES, bool GHOST, int MINB, int RECON, int NRHS = 1, int RHSL = 1,
          bool VBLK = false>
__global__ void __launch_bounds__(256, MINB) dslash_kernel(const StencilParams P) {
    // every block has started: the next PDL-launched apply may begin filling freed SMs
    asm volatile("griddepcontrol.launch_dependents;");
    dslash_body<LR, VR, LANES, GHOST, RECON, NRHS, RHSL, false, VBLK>(P, (int64_t)blockIdx.x * blockDim.x + threadIdx.x,
                                                                     P.box_start[P.nbox]);
}

// The neighbour-staged variant (DSLASH_OPT_STAGE): one tile of P.stage_ty full x-rows per block
// (blockDim = lxh * stage_ty * LANES * RHSL threads), the tile's source rows y0-3 .. y0+TY+2 in
// dynamic shared memory (NRHS * RHSL * 3 * (TY + 6) * lxh complex).  Boxes span full x and y, so
// tiles never straddle a box and every thread is valid.
template <typename LR, typename VR, int LANES, bool GHOST, int RECON, int NRHS = 1, int RHSL = 1>
__global__ void __launch_bounds__(256, 2) dslash_stage_kernel(const StencilParams P) {
    using V2 = cplx_t<VR>;
    asm volatile("griddepcontrol.launch_dependents;");
    __shared__ uint64_t bar;
    extern __shared__ __align__(128) unsigned char stage_smem[];
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int64_t tile_sites = (int64_t)P.lxh * P.stage_ty;
    const Site s0 = decode_site(P, (int64_t)blockIdx.x * tile_sites);
    StageTile<V2> T;
    T.sv = reinterpret_cast<V2*>(stage_smem);
    T.bar = &bar;
    T.y0 = s0.y;
    T.rows = P.stage_ty + 6;
    T.plane0 = s0.cb - s0.xh - (int64_t)P.lxh * s0.y;
    T.sbase = smem_addr(stage_smem);
    dslash_body<LR, VR, LANES, GHOST, RECON, NRHS, RHSL, true>(P, (int64_t)blockIdx.x * blockDim.x + threadIdx.x,
                                                               P.box_start[P.nbox], T);
}

}  // namespace hisq
