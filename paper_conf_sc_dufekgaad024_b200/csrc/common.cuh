// common.cuh -- shared device-side types and PTX helpers for the HISQ Dslash kernels (sm_100a).
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace hisq {

// ---------------------------------------------------------------- fast unsigned division
// q = n / d for 0 <= n < 2^31 and d >= 1 via one mul.hi: the round-up magic-number division of
// Granlund & Montgomery, "Division by invariant integers using multiplication" (PLDI 1994, §4),
// m = 2^32 (2^s - d) / d + 1, q = (umulhi(n, m) + n) >> s with s = ceil(log2 d).
struct FastDiv {
    uint32_t d, m, s;
    __host__ void init(uint32_t div) {
        d = div;
        s = 0;
        while ((1ull << s) < div) ++s;
        m = (uint32_t)((((1ull << 32) * ((1ull << s) - div)) / div) + 1);
    }
    __device__ __forceinline__ uint32_t div(uint32_t n) const {
        return (uint32_t)(((uint64_t)__umulhi(n, m) + n) >> s);
    }
};

// ---------------------------------------------------------------- cache-policy loads/stores
// Links are streamed exactly once: keep them out of L1 and mark their L2 lines evict-first so
// the reused source vectors (16 consumers each) stay L2-resident.
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}

__device__ __forceinline__ double2 ld_stream(const double2* p, uint64_t pol) {
    double2 r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;"
        : "=d"(r.x), "=d"(r.y)
        : "l"(p), "l"(pol));
    return r;
}

__device__ __forceinline__ double2 ld_reuse(const double2* p, uint64_t pol) {
    double2 r;
    asm("ld.global.nc.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;" : "=d"(r.x), "=d"(r.y) : "l"(p), "l"(pol));
    return r;
}

// a reused vector that THIS SM will not read again (the z / t hops: their other consumers run on
// other SMs): L2 evict_last like ld_reuse, but no L1 line, so it does not evict the x / y rows
// the block's own threads reuse
__device__ __forceinline__ double2 ld_reuse_na(const double2* p, uint64_t pol) {
    double2 r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;" : "=d"(r.x), "=d"(r.y) : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ float2 ld_reuse_na(const float2* p, uint64_t pol) {
    float2 r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f32 {%0, %1}, [%2], %3;" : "=f"(r.x), "=f"(r.y) : "l"(p), "l"(pol));
    return r;
}

__device__ __forceinline__ void st_stream(double2* p, double2 v) {
    asm volatile("st.global.cs.v2.f64 [%0], {%1, %2};" ::"l"(p), "d"(v.x), "d"(v.y) : "memory");
}

__device__ __forceinline__ float2 ld_stream(const float2* p, uint64_t pol) {
    float2 r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f32 {%0, %1}, [%2], %3;"
        : "=f"(r.x), "=f"(r.y)
        : "l"(p), "l"(pol));
    return r;
}

__device__ __forceinline__ float4 ld_stream(const float4* p, uint64_t pol) {
    float4 r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
        : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
        : "l"(p), "l"(pol));
    return r;
}

__device__ __forceinline__ float2 ld_reuse(const float2* p, uint64_t pol) {
    float2 r;
    asm("ld.global.nc.L2::cache_hint.v2.f32 {%0, %1}, [%2], %3;" : "=f"(r.x), "=f"(r.y) : "l"(p), "l"(pol));
    return r;
}

__device__ __forceinline__ void st_stream(float2* p, float2 v) {
    asm volatile("st.global.cs.v2.f32 [%0], {%1, %2};" ::"l"(p), "f"(v.x), "f"(v.y) : "memory");
}

// ---------------------------------------------------------------- mbarrier / bulk-copy PTX
__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}" ::"r"(smem_addr(bar)),
        "r"(parity)
        : "memory");
}
// global -> shared bulk copy (TMA engine), completion signalled on `bar` as transaction bytes
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::
            "r"(smem_addr(dst)),
        "l"(src), "r"(bytes), "r"(smem_addr(bar)), "l"(pol)
        : "memory");
}

__device__ __forceinline__ double2 lds(const double2* p) {
    double2 r;
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(r.x), "=d"(r.y) : "r"(smem_addr(p)));
    return r;
}
__device__ __forceinline__ float2 lds(const float2* p) {
    float2 r;
    asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(r.x), "=f"(r.y) : "r"(smem_addr(p)));
    return r;
}

// ---------------------------------------------------------------- precision
// complex type of a real type: cplx_t<double> = double2, cplx_t<float> = float2
template <typename R> struct CplxOf;
template <> struct CplxOf<double> { using type = double2; };
template <> struct CplxOf<float> { using type = float2; };
template <typename R> using cplx_t = typename CplxOf<R>::type;

template <typename T> __device__ __forceinline__ T to_cplx(double2 v);
template <> __device__ __forceinline__ double2 to_cplx<double2>(double2 v) { return v; }
template <> __device__ __forceinline__ float2 to_cplx<float2>(double2 v) {
    return make_float2((float)v.x, (float)v.y);
}
__device__ __forceinline__ double2 widen(double2 v) { return v; }
__device__ __forceinline__ double2 widen(float2 v) { return make_double2(v.x, v.y); }

// ---------------------------------------------------------------- complex fp64 arithmetic
// acc += a * b
__device__ __forceinline__ void cmadd(double2& acc, double2 a, double2 b) {
    acc.x = fma(a.x, b.x, acc.x);
    acc.x = fma(-a.y, b.y, acc.x);
    acc.y = fma(a.x, b.y, acc.y);
    acc.y = fma(a.y, b.x, acc.y);
}
// acc -= a * b
__device__ __forceinline__ void cmsub(double2& acc, double2 a, double2 b) {
    acc.x = fma(-a.x, b.x, acc.x);
    acc.x = fma(a.y, b.y, acc.x);
    acc.y = fma(-a.x, b.y, acc.y);
    acc.y = fma(-a.y, b.x, acc.y);
}
__device__ __forceinline__ void cmadd(float2& acc, float2 a, float2 b) {
    acc.x = fmaf(a.x, b.x, acc.x);
    acc.x = fmaf(-a.y, b.y, acc.x);
    acc.y = fmaf(a.x, b.y, acc.y);
    acc.y = fmaf(a.y, b.x, acc.y);
}
__device__ __forceinline__ void cmsub(float2& acc, float2 a, float2 b) {
    acc.x = fmaf(-a.x, b.x, acc.x);
    acc.x = fmaf(a.y, b.y, acc.x);
    acc.y = fmaf(-a.x, b.y, acc.y);
    acc.y = fmaf(-a.y, b.x, acc.y);
}

// ---------------------------------------------------------------- double-double sums
// The solver's dot products are accumulated as unevaluated sums hi + lo (Dekker / Knuth TwoSum,
// "double-double"), at every level: per thread, per block, over the blocks and over the ranks.
// The rounded result hi is then the correctly rounded sum of the (bitwise identical, element-wise)
// terms unless that exact sum lies within ~n u^2 |sum| of a rounding boundary, so it no longer
// depends on how the lattice is split over ranks (DESIGN.md §12 f-3): a P-rank CG runs the
// 1-rank iterates bit for bit.  Operands are combined with explicit __dadd_rn / __dsub_rn, which
// the compiler never contracts or reassociates.
__device__ __forceinline__ double2 two_sum(double a, double b) {
    const double s = __dadd_rn(a, b);
    const double bb = __dsub_rn(s, a);
    const double e = __dadd_rn(__dsub_rn(a, __dsub_rn(s, bb)), __dsub_rn(b, bb));
    return make_double2(s, e);
}
// x + t (t a double); renormalised with TwoSum (no |a| >= |b| precondition, so cancellation is safe)
__device__ __forceinline__ double2 dd_add(double2 x, double t) {
    const double2 s = two_sum(x.x, t);
    return two_sum(s.x, __dadd_rn(s.y, x.y));
}
// x + y (both double-double; the low parts are added with TwoSum too).  Symmetric in x and y
// (TwoSum's error term is exact), so a shuffle butterfly gives every lane the same bits.
__device__ __forceinline__ double2 dd_add(double2 x, double2 y) {
    const double2 s = two_sum(x.x, y.x);
    const double2 t = two_sum(x.y, y.y);
    const double2 u = two_sum(s.x, __dadd_rn(s.y, t.x));
    return two_sum(u.x, __dadd_rn(u.y, t.y));
}
// Re(conj(a) b) of one complex element, in one fixed expression (the same bits in every kernel)
__device__ __forceinline__ double dot_term(double2 a, double2 b) { return __fma_rn(a.x, b.x, __dmul_rn(a.y, b.y)); }
__device__ __forceinline__ double dot_term(float2 a, float2 b) {
    return __fma_rn((double)a.x, (double)b.x, __dmul_rn((double)a.y, (double)b.y));
}

// ---------------------------------------------------------------- kernel parameters
constexpr int kMaxBoxes = 5;  // interior + up to 4 boundary slabs (t and z halo)

struct Box {
    int lo[4];
    int n[4];  // extent per dim; n[0] counts full x extent (sites per row = n[0] / 2)
};

// Pointers are untyped: the kernel instantiation fixes the link type (double2 or float2) and
// the vector type (double2 or float2).
struct StencilParams {
    const void* links;         // internal link layout for the target parity (variant-specific)
    const void* in;            // [3][vh] source parity, local
    void* out;                 // [3][vh] target parity, local
    const void* ghost[4][2];   // [mu][side] -> [3][face_vh[mu]] (only where halo[mu])
    int64_t vh;
    int64_t face_vh[4];
    double long_inv_scale;     // 1/s of the long links N = s W (recon-12 only)
    double long_scale;         // s of the long links N = s e^{i psi} W (recon-9 only)
    int L[4];                  // local extents
    int lxh;                   // L[0] / 2
    int parity;                // (target parity + origin sum) & 1, origin sum is even -> target parity
    int halo_mask;             // bit mu set: direction mu reads ghosts outside [0, L[mu])
    int nbox;
    Box box[kMaxBoxes];
    int64_t box_start[kMaxBoxes + 1];  // prefix sum of target sites per box
    FastDiv div_xh[kMaxBoxes], div_y[kMaxBoxes], div_z[kMaxBoxes];
    int stage_ty;              // rows per tile of the neighbour-staged kernel (DSLASH_OPT_STAGE)
    int halo_pass;             // GHOST kernels: kPassAll, or one pass of the split-by-direction overlap
    // producer push (DSLASH_OPT_PUSH; GHOST kernels only): a target site within 3 slices of the
    // bottom (top) of a direction mu in push_mask also stores its output into push[mu][0] ([mu][1]):
    // the minus (plus) neighbour's plus (minus) ghost face, [3][face_vh[mu]], peer memory over NVLink
    void* push[4][2];
    int push_mask;
    // site-blocked vectors (VBLK kernels): complex elements per 16-site block = 16 * 3 * nrhs of
    // the whole apply (a launch of NRHS right-hand sides starts at its first one's rows)
    int64_t vblk;
};

// Passes of a GHOST kernel (StencilParams::halo_pass).  kPassAll reads local sources and ghost
// faces alike.  The split-by-direction overlap (DSLASH_OVERLAP_DIRS) runs kPassLocal over every
// site while the faces are in flight (hops into a ghost face are skipped, link and vector), then
// kPassGhost over the boundary sites: only the skipped hops, added to the stored partial sum.
constexpr int kPassAll = 0, kPassLocal = 1, kPassGhost = 2;

}  // namespace hisq
