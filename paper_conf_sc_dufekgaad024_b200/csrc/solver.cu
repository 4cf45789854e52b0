// solver.cu -- the even-odd normal operator and a conjugate-gradient solver on top of the
// single-parity Dslash ("both-parity D^dag D = -D_oe D_eo, plus CG", the step
// downstream of the Dslash in su3_rhmd_hisq).
//
// With D anti-Hermitian (D_{p,1-p} = -D_{1-p,p}^dag, pin P3), the operator
//     A_p = m^2 - D_{p,1-p} D_{1-p,p} = m^2 + D_{1-p,p}^dag D_{1-p,p}
// is Hermitian positive definite on parity p for m != 0, and CG solves A_p x = b.
// Dot products are accumulated as double-double sums at every level (thread, block, grid, ranks;
// common.cuh) and rounded once, so they do not depend on the decomposition: with several ranks
// the per-rank sums are all-gathered (ncclAllGather, or the P2P transport's IPC-mapped slots)
// and every rank adds them in rank order, the solver's one true collective.
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>

#include "common.cuh"
#include "handle.h"

namespace {

using hisq::dd_add;
using hisq::dot_term;

constexpr int kRedThreads = 256;
constexpr int kRedBlocks = 592;  // 4 x 148 SMs; fixed, so the summation order never changes

// block-level double-double sum of v (all threads call); result valid in thread 0
__device__ double2 block_sum(double2 v) {
    __shared__ double2 warp_part[kRedThreads / 32];
#pragma unroll
    for (int off = 16; off; off >>= 1)
        v = dd_add(v, make_double2(__shfl_xor_sync(0xffffffffu, v.x, off), __shfl_xor_sync(0xffffffffu, v.y, off)));
    if ((threadIdx.x & 31) == 0) warp_part[threadIdx.x >> 5] = v;
    __syncthreads();
    double2 s = make_double2(0.0, 0.0);
    if (threadIdx.x == 0)
        for (int w = 0; w < kRedThreads / 32; ++w) s = dd_add(s, warp_part[w]);
    return s;
}

// Vector kernels, templated on the complex type (double2: the fp64 solver; float2: the inner
// solver of dslash_cg_mixed).  Dot products accumulate in fp64 whatever the vector type.

// q = m2 p - q ; partial[block] = sum Re(conj(p) q)
template <typename V2>
__global__ void __launch_bounds__(kRedThreads) k_normal_finish(const V2* __restrict__ p, V2* __restrict__ q,
                                                               double m2, int64_t n, double2* __restrict__ partial) {
    using R = decltype(V2{}.x);
    double2 acc = make_double2(0.0, 0.0);
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const V2 a = p[i];
        V2 b = q[i];
        b.x = (R)m2 * a.x - b.x;
        b.y = (R)m2 * a.y - b.y;
        q[i] = b;
        acc = dd_add(acc, dot_term(a, b));
    }
    const double2 s = block_sum(acc);
    if (partial && threadIdx.x == 0) partial[blockIdx.x] = s;
}

// partial[block] = sum |v|^2
template <typename V2>
__global__ void __launch_bounds__(kRedThreads) k_norm2(const V2* __restrict__ v, int64_t n,
                                                       double2* __restrict__ partial) {
    double2 acc = make_double2(0.0, 0.0);
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const V2 a = v[i];
        acc = dd_add(acc, dot_term(a, a));
    }
    const double2 s = block_sum(acc);
    if (threadIdx.x == 0) partial[blockIdx.x] = s;
}

// x += alpha p ; r -= alpha q ; partial[block] = sum |r|^2, alpha = rr / pq read on the device
// (0 when pq == 0, or once rr <= stop: an iterate that converged stays put through the iterations
// the host queued before it saw the convergence)
template <typename V2>
__global__ void __launch_bounds__(kRedThreads) k_cg_update(V2* __restrict__ x, V2* __restrict__ r,
                                                           const V2* __restrict__ p, const V2* __restrict__ q,
                                                           const double* __restrict__ rr, const double* __restrict__ pq,
                                                           double stop, int64_t n, double2* __restrict__ partial) {
    using R = decltype(V2{}.x);
    const R alpha = (R)((*pq != 0.0 && *rr > stop) ? *rr / *pq : 0.0);
    double2 acc = make_double2(0.0, 0.0);
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        V2 xi = x[i], ri = r[i];
        const V2 pi = p[i], qi = q[i];
        xi.x = fma(alpha, pi.x, xi.x);
        xi.y = fma(alpha, pi.y, xi.y);
        ri.x = fma(-alpha, qi.x, ri.x);
        ri.y = fma(-alpha, qi.y, ri.y);
        x[i] = xi;
        r[i] = ri;
        acc = dd_add(acc, dot_term(ri, ri));
    }
    const double2 s = block_sum(acc);
    if (threadIdx.x == 0) partial[blockIdx.x] = s;
}

// sum of the kRedBlocks block partials in k_finalize's order (every block of kRedThreads threads
// gets the same bits); result valid in thread 0
// (coherent L2 loads: in the fused CG step other blocks wrote the partials during this launch)
__device__ __forceinline__ double2 sum_partials(const double2* partial, int n) {
    double2 acc = make_double2(0.0, 0.0);
    for (int k = threadIdx.x; k < n; k += kRedThreads) acc = dd_add(acc, __ldcg(partial + k));
    return block_sum(acc);
}

// element i = c * vh + cb of a [3][vh] vector: also store it into the pushed ghost faces its site
// belongs to (F.mask != 0; the face order of the stencil kernel's push, stencil.cuh)
template <typename V2>
__device__ __forceinline__ void push_element(const FacePush& F, int64_t i, V2 v) {
    const int64_t c = i / F.vh, cb = i - c * F.vh;
    const int64_t zrow = (int64_t)F.lxh * F.L1, tslab = zrow * F.L2;
    const int t = (int)(cb / tslab);
    if (F.mask & 8) {
        const int64_t fv = F.face_vh[3];
        if (t < 3) static_cast<V2*>(F.dst[3][0])[c * fv + cb] = v;
        if (t >= F.L3 - 3) static_cast<V2*>(F.dst[3][1])[c * fv + cb - (int64_t)(F.L3 - 3) * tslab] = v;
    }
    if (F.mask & 4) {
        const int64_t fv = F.face_vh[2];
        const int64_t in_row = cb % zrow;
        const int z = (int)((cb / zrow) % F.L2);
        if (z < 3) static_cast<V2*>(F.dst[2][0])[c * fv + in_row + zrow * (z + 3 * (int64_t)t)] = v;
        if (z >= F.L2 - 3)
            static_cast<V2*>(F.dst[2][1])[c * fv + in_row + zrow * (z - (F.L2 - 3) + 3 * (int64_t)t)] = v;
    }
}

// p = r + beta p, beta = rr_new / rr read on the device (0 when rr == 0); with the producer push the
// faces of the new p go straight to the neighbours' ghosts for the next iteration's first apply
template <typename V2>
__global__ void k_cg_direction(V2* __restrict__ p, const V2* __restrict__ r, const double* __restrict__ rr_new,
                               const double* __restrict__ rr, int64_t n, const FacePush F) {
    using R = decltype(V2{}.x);
    const R beta = (R)((*rr != 0.0) ? *rr_new / *rr : 0.0);
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const V2 ri = r[i];
        V2 pi = p[i];
        pi.x = fma(beta, pi.x, ri.x);
        pi.y = fma(beta, pi.y, ri.y);
        p[i] = pi;
        if (F.mask) push_element(F, i, pi);
    }
}

// grid barrier of a cooperative launch (thread 0 of every block): publish this block's writes,
// arrive, wait until the monotonic counter reaches `target`
__device__ __forceinline__ void grid_arrive_wait(unsigned long long* bar, unsigned long long target) {
    __threadfence();
    atomicAdd(bar, 1ull);
    unsigned long long v;
    do {
        asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(bar) : "memory");
    } while (v < target);
}

// One CG step after q = A p (one rank, cooperative launch of kRedBlocks co-resident blocks):
//   q = m2 p - q ; <p, q> partials -> partial ; grid barrier          (k_normal_finish)
//   pq = sum(partial)                       (k_finalize)
//   x += alpha p ; r -= alpha q ; |r|^2 partials -> partial2           (k_cg_update)
//   grid barrier
//   rr_new = sum(partial2) ; p = r + beta p (+ face push)              (k_finalize, k_cg_direction)
// with the same per-element arithmetic, grid and reduction order as those four kernels, so the
// iterates are bitwise the unfused ones; three launches and their gaps fewer, and r, p are
// re-read from L2.  The barrier counter is monotonic: this launch's blocks wait for `target`.
template <typename V2>
__global__ void __launch_bounds__(kRedThreads) k_cg_step(V2* __restrict__ x, V2* __restrict__ r, V2* __restrict__ p,
                                                         V2* __restrict__ q, double m2, const double* __restrict__ rr,
                                                         double* __restrict__ pq_out, double* __restrict__ rr_new_out,
                                                         double stop, int64_t n, double2* partial,
                                                         double2* partial2, unsigned long long* bar,
                                                         unsigned long long target, double* rr_host,
                                                         const FacePush F) {
    using R = decltype(V2{}.x);
    __shared__ double s_val;
    {  // q = m2 p - q and the <p, q> block partials (k_normal_finish), then a grid barrier
        double2 acc0 = make_double2(0.0, 0.0);
        for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
            const V2 a = p[i];
            V2 b = q[i];
            b.x = (R)m2 * a.x - b.x;
            b.y = (R)m2 * a.y - b.y;
            q[i] = b;
            acc0 = dd_add(acc0, dot_term(a, b));
        }
        const double2 s = block_sum(acc0);
        if (threadIdx.x == 0) {
            partial[blockIdx.x] = s;
            grid_arrive_wait(bar, target - kRedBlocks);
        }
        __syncthreads();
    }
    const double s0 = sum_partials(partial, kRedBlocks).x;   // one rank: the rounded sum is hi
    if (threadIdx.x == 0) s_val = s0;
    __syncthreads();
    const double pq = s_val;
    if (blockIdx.x == 0 && threadIdx.x == 0) *pq_out = pq;
    const double rrv = *rr;
    const R alpha = (R)((pq != 0.0 && rrv > stop) ? rrv / pq : 0.0);
    double2 acc = make_double2(0.0, 0.0);
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        V2 xi = x[i], ri = r[i];
        const V2 pi = p[i], qi = q[i];
        xi.x = fma(alpha, pi.x, xi.x);
        xi.y = fma(alpha, pi.y, xi.y);
        ri.x = fma(-alpha, qi.x, ri.x);
        ri.y = fma(-alpha, qi.y, ri.y);
        x[i] = xi;
        r[i] = ri;
        acc = dd_add(acc, dot_term(ri, ri));
    }
    const double2 s1 = block_sum(acc);
    if (threadIdx.x == 0) {
        partial2[blockIdx.x] = s1;
        grid_arrive_wait(bar, target);
    }
    __syncthreads();
    const double s2 = sum_partials(partial2, kRedBlocks).x;
    __syncthreads();  // s_val is reused
    if (threadIdx.x == 0) s_val = s2;
    __syncthreads();
    const double rr_new = s_val;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *rr_new_out = rr_new;
        if (rr_host) {  // the host's copy, through the mapped pinned buffer (no copy in the stream)
            *(volatile double*)rr_host = rr_new;
            __threadfence_system();
        }
    }
    const R beta = (R)((rrv != 0.0) ? rr_new / rrv : 0.0);
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const V2 ri = r[i];
        V2 pi = p[i];
        pi.x = fma(beta, pi.x, ri.x);
        pi.y = fma(beta, pi.y, ri.y);
        p[i] = pi;
        if (F.mask) push_element(F, i, pi);
    }
}

// dslash_cg_mixed: r32 = (float) r ; x += (double) e32
__global__ void k_round_to_f32(float2* __restrict__ o, const double2* __restrict__ v, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        o[i] = make_float2((float)v[i].x, (float)v[i].y);
}
__global__ void k_add_f32(double2* __restrict__ x, const float2* __restrict__ e, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        double2 xi = x[i];
        xi.x += (double)e[i].x;
        xi.y += (double)e[i].y;
        x[i] = xi;
    }
}

// r = b - r  (true residual from r = A x)
__global__ void k_sub_from(double2* __restrict__ r, const double2* __restrict__ b, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const double2 bi = b[i];
        double2 ri = r[i];
        ri.x = bi.x - ri.x;
        ri.y = bi.y - ri.y;
        r[i] = ri;
    }
}

// The rank's double-double sum of the n block partials (thread t adds k = t, t + 256, ... in order,
// then the fixed shuffle tree of block_sum): *dd_out (for the cross-rank sum) and, with one rank,
// the rounded result *out = hi (out may be NULL)
__global__ void __launch_bounds__(kRedThreads) k_finalize(const double2* __restrict__ partial, int n,
                                                          double2* __restrict__ dd_out, double* __restrict__ out) {
    double2 acc = make_double2(0.0, 0.0);
    for (int k = threadIdx.x; k < n; k += kRedThreads) acc = dd_add(acc, partial[k]);
    const double2 s = block_sum(acc);
    if (threadIdx.x == 0) {
        *dd_out = s;
        if (out) *out = s.x;
    }
}

// *out = the rounded sum of the ranks' double-double sums v[0..n), added in rank order (every rank
// runs this on the same gathered values: the same bits everywhere)
__global__ void k_rank_sum(const double2* __restrict__ v, int n, double* __restrict__ out) {
    double2 acc = make_double2(0.0, 0.0);
    for (int r = 0; r < n; ++r) acc = dd_add(acc, v[r]);
    *out = acc.x;
}

}  // namespace

// ---------------------------------------------------------------------------- host helpers
static int num_sms_solver() {
    static int n = 0;
    int dev = 0;
    if (!n && (cudaGetDevice(&dev) != cudaSuccess ||
               cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess))
        n = 148;
    return n;
}

static dslash_status need_scratch(dslash_t h) {
    const size_t bytes = 3 * (size_t)h->plan.vh_local * sizeof(double2);
    for (void*& v : h->cg_vec)
        if (!v) CU(h, cudaMalloc(&v, bytes));
    if (!h->cg_partial) CU(h, cudaMalloc(&h->cg_partial, kRedBlocks * sizeof(double2)));
    if (!h->cg_partial2) CU(h, cudaMalloc(&h->cg_partial2, kRedBlocks * sizeof(double2)));
    if (!h->cg_dd) CU(h, cudaMalloc(&h->cg_dd, (1 + kMaxRanks) * sizeof(double2)));
    if (!h->cg_bar) {
        CU(h, cudaMalloc(&h->cg_bar, sizeof(unsigned long long)));
        CU(h, cudaMemset(h->cg_bar, 0, sizeof(unsigned long long)));
        h->cg_bar_next = 0;
    }
    if (!h->cg_scalar) CU(h, cudaMalloc(&h->cg_scalar, 4 * sizeof(double)));
    return DSLASH_OK;
}

// the partials of one reduction -> global sum over all ranks in device scalar `slot`: this rank's
// double-double sum, then (several ranks) an all-gather of every rank's and their sum in rank
// order.  NCCL groups gather with ncclAllGather; the P2P transport (no communicator, e.g. several
// ranks on one GPU) through the ranks' IPC-mapped control blocks (hisq_p2p_gather).
static dslash_status reduce_to_slot(dslash_t h, cudaStream_t s, double* slot) {
    const int n = h->plan.nranks;
    k_finalize<<<1, kRedThreads, 0, s>>>(h->cg_partial, kRedBlocks, h->cg_dd, n == 1 ? slot : nullptr);
    CU(h, cudaGetLastError());
    if (n == 1) return DSLASH_OK;
    const double2* all = h->cg_dd + 1;
    if (h->nccl) {
        NC(h, ncclAllGather(h->cg_dd, h->cg_dd + 1, 2, ncclDouble, h->nccl, s));
    } else {
        dslash_status st = hisq_p2p_gather(h, s, h->cg_dd, &all);
        if (st != DSLASH_OK) return st;
    }
    k_rank_sum<<<1, 1, 0, s>>>(all, n, slot);
    CU(h, cudaGetLastError());
    return DSLASH_OK;
}

// ... and to the host (synchronous)
static dslash_status reduce_to_host(dslash_t h, cudaStream_t s, double* value) {
    dslash_status st = reduce_to_slot(h, s, h->cg_scalar);
    if (st != DSLASH_OK) return st;
    CU(h, cudaMemcpyAsync(value, h->cg_scalar, sizeof(double), cudaMemcpyDeviceToHost, s));
    CU(h, cudaStreamSynchronize(s));
    return DSLASH_OK;
}

static dslash_status check_solver_args(dslash_t h, const void* a, const void* b, int32_t parity,
                                       bool reduces = true) {
    if (!h) return hisq_fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (parity & ~1) return hisq_fail(h, DSLASH_ERR_ARG, "parity %d not in {0,1}", parity);
    if (h->parity_mask != DSLASH_BOTH)
        return hisq_fail(h, DSLASH_ERR_ARG, "the normal operator applies both parities: create with DSLASH_BOTH");
    if (h->precision == DSLASH_F32)
        return hisq_fail(h, DSLASH_ERR_UNSUPPORTED, "the solver works on fp64 vectors (DSLASH_F64 or DSLASH_MIXED)");
    if (!h->loaded) return hisq_fail(h, DSLASH_ERR_STATE, "solver before load_links");
    if (reduces && h->plan.nranks > 1 && !h->nccl && h->transport != DSLASH_TRANSPORT_P2P)
        return hisq_fail(h, DSLASH_ERR_UNSUPPORTED, "dot products across ranks need NCCL or the P2P transport");
    if (h->plan.nranks > kMaxRanks)
        return hisq_fail(h, DSLASH_ERR_UNSUPPORTED, "the solver sums over at most %d ranks", kMaxRanks);
    if (!a || !b || ((uintptr_t)a & 15) || ((uintptr_t)b & 15))
        return hisq_fail(h, DSLASH_ERR_ARG, "NULL or misaligned vector");
    const uintptr_t n = 3 * (uintptr_t)h->plan.vh_local * sizeof(double2);
    if ((uintptr_t)a < (uintptr_t)b + n && (uintptr_t)b < (uintptr_t)a + n)
        return hisq_fail(h, DSLASH_ERR_ARG, "vectors overlap");
    return DSLASH_OK;
}

// q = A p, and (if partial) the block partials of Re<p, q>
template <typename V2>
static dslash_status normal_apply(dslash_t h, V2* q, const V2* p, int32_t parity, double m2, V2* tmp, cudaStream_t s,
                                  bool dot, bool finish = true) {
    // t = D_{1-p,p} p; with the producer push its faces go straight to the neighbours' ghosts
    dslash_status st = hisq_apply(h, tmp, p, 1 - parity, 1, s, h->push != 0);
    if (st != DSLASH_OK) return st;
    if ((st = hisq_apply(h, q, tmp, parity, 1, s)) != DSLASH_OK) return st;  // q = D_{p,1-p} t
    if (!finish) return DSLASH_OK;  // the caller's kernel applies q = m^2 p - q (fused CG step)
    const int64_t n = 3 * h->plan.vh_local;
    k_normal_finish<<<kRedBlocks, kRedThreads, 0, s>>>(p, q, m2, n, dot ? h->cg_partial : nullptr);
    CU(h, cudaGetLastError());
    return DSLASH_OK;
}

extern "C" dslash_status dslash_normal_apply(dslash_t h, void* out, const void* in, int32_t parity, double mass,
                                             dslash_stream_t stream) {
    DeviceGuard device_guard(h);
    dslash_status st = check_solver_args(h, out, in, parity, false);  // no dot product
    if (st != DSLASH_OK) return st;
    if ((st = need_scratch(h)) != DSLASH_OK) return st;
    return normal_apply(h, (double2*)out, (const double2*)in, parity, mass * mass, (double2*)h->cg_vec[3],
                        (cudaStream_t)stream, false);
}

// CG iterations on A x = b from x = 0, r = p = b (the caller set them up): standard
// Hestenes-Stiefel recurrences, run until <r, r> <= stop or max_iter.  Device scalars: sc[0], sc[1] =
// <r,r> of alternate iterations (ping-pong, so no kernel overwrites a value another block may
// still read), sc[2] = <p, A p>; sc[0] must hold <b, b> on entry.  The host learns <r,r> through
// pinned memory kCgLag iterations late, so the GPU never waits for the host and the host's
// enqueue jitter is absorbed by a queue several iterations deep.  The iterations queued past
// convergence are frozen on the device (k_cg_update takes alpha = 0 once <r,r> <= stop), so x is
// exactly the first converged iterate and *iters its index.  V2 = double2 (fp64) or float2 (the
// inner solve of dslash_cg_mixed, on the fp32 links).
constexpr int kCgLag = 3;

template <typename V2>
static dslash_status cg_core(dslash_t h, V2* x, V2* r, V2* p, V2* q, V2* t, int32_t parity, double m2, double stop,
                             int32_t max_iter, cudaStream_t s, int32_t* iters, double* rr_last, bool* converged) {
    const int64_t n = 3 * h->plan.vh_local;
    double* sc = h->cg_scalar;
    static_assert(kCgLag + 1 <= (int)(sizeof(dslash_s::cg_ev) / sizeof(cudaEvent_t)), "event ring");
    cudaEvent_t* ev = h->cg_ev;
    dslash_status st = DSLASH_OK;
    auto release = [&]() {};
#define CUR(call)                                                                                    \
    do {                                                                                             \
        cudaError_t e_ = (call);                                                                     \
        if (e_ != cudaSuccess) {                                                                     \
            release();                                                                               \
            return hisq_fail(h, DSLASH_ERR_CUDA, "%s:%d %s: %s", __FILE__, __LINE__, #call,          \
                             cudaGetErrorString(e_));                                                \
        }                                                                                            \
    } while (0)
    int need = (max_iter < 1 ? 1 : max_iter) + 1;
    if (h->cg_host_cap < need) {
        need = need < 2 * h->cg_host_cap ? 2 * h->cg_host_cap : need < 8192 ? 8192 : need;
        if (h->cg_host_rr) CUR(cudaFreeHost(h->cg_host_rr));
        h->cg_host_rr = nullptr;
        h->cg_host_cap = 0;
        CUR(cudaMallocHost(&h->cg_host_rr, (size_t)need * sizeof(double)));
        h->cg_host_cap = need;
    }
    double* host_rr = h->cg_host_rr;  // host_rr[k] = <r,r> after iteration k
    double* host_rr_dev = nullptr;     // its device alias (pinned host memory is mapped under UVA)
    CUR(cudaHostGetDevicePointer((void**)&host_rr_dev, host_rr, 0));
    host_rr[0] = HUGE_VAL;            // (max_iter < 1: no iteration, not converged)
    for (int i = 0; i <= kCgLag; ++i)
        if (!ev[i]) CUR(cudaEventCreateWithFlags(&ev[i], cudaEventDisableTiming));
    *converged = false;
    int k = 0, kstar = 0;  // last enqueued iteration; first converged one (0: none seen yet)
    // fused CG step: one rank (no cross-rank sum between the update and the direction), and all
    // kRedBlocks blocks co-resident (probed once per handle); HISQ_CG_UNFUSED=1 forces the
    // four-kernel path
    if (h->cg_fused < 0) {
        int occ = 0, dev = 0, coop = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, dev);
        const bool ok = coop &&
                        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_cg_step<double2>, kRedThreads, 0) ==
                            cudaSuccess &&
                        occ * num_sms_solver() >= kRedBlocks;
        int occ32 = 0;
        const bool ok32 = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ32, k_cg_step<float2>, kRedThreads, 0) ==
                              cudaSuccess &&
                          occ32 * num_sms_solver() >= kRedBlocks;
        cudaGetLastError();
        h->cg_fused = (ok && ok32 && !getenv("HISQ_CG_UNFUSED")) ? 1 : 0;
    }
    const bool fused = h->cg_fused == 1 && h->plan.nranks == 1;
    // HISQ_CG_PROFILE=1: host time per iteration spent enqueueing vs waiting, to stderr
    static const bool prof = getenv("HISQ_CG_PROFILE") != nullptr;
    using clk = std::chrono::steady_clock;
    double enq_us = 0.0, enq_max = 0.0, wait_us = 0.0;
    for (k = 1; k <= max_iter; ++k) {
        const auto t0 = prof ? clk::now() : clk::time_point{};
        double* rr_cur = &sc[(k - 1) & 1];
        double* rr_new = &sc[k & 1];
        // q = A p (with the fused step, q = D D p here and m^2 p - q inside the step kernel)
        if ((st = normal_apply(h, q, p, parity, m2, t, s, true, !fused)) != DSLASH_OK) break;
        if (fused) {  // one rank: the rest of the step in one cooperative launch
            FacePush fp;
            if ((st = hisq_push_begin(h, s, &fp)) != DSLASH_OK) break;
            // the counter only advances once the launch is accepted (a refused launch must not
            // leave the next one waiting for arrivals that never come)
            unsigned long long target = h->cg_bar_next + 2 * kRedBlocks;  // two barriers per launch
            double m2_v = m2;
            double stop_v = stop;
            int64_t n_v = n;
            double* pq_slot = &sc[2];
            const double* rr_c = rr_cur;
            double2* part = h->cg_partial;
            double2* part2 = h->cg_partial2;
            unsigned long long* bar = h->cg_bar;
            double* rr_host = host_rr_dev + k;  // host_rr[k], written by the kernel
            void* args[] = {&x,    &r,    &p,     &q,   &m2_v,   &rr_c,    &pq_slot, &rr_new,
                            &stop_v, &n_v, &part, &part2, &bar, &target, &rr_host, &fp};
            CUR(cudaLaunchCooperativeKernel((const void*)k_cg_step<V2>, kRedBlocks, kRedThreads, args, 0, s));
            h->cg_bar_next = target;
            if ((st = hisq_push_end(h, s, p)) != DSLASH_OK) break;
        } else {
        if ((st = reduce_to_slot(h, s, &sc[2])) != DSLASH_OK) break;                 // <p, q>
        k_cg_update<<<kRedBlocks, kRedThreads, 0, s>>>(x, r, p, q, rr_cur, &sc[2], stop, n, h->cg_partial);
        CUR(cudaGetLastError());
        if ((st = reduce_to_slot(h, s, rr_new)) != DSLASH_OK) break;                  // <r, r>
        FacePush fp;
        if ((st = hisq_push_begin(h, s, &fp)) != DSLASH_OK) break;
        k_cg_direction<<<kRedBlocks, kRedThreads, 0, s>>>(p, r, rr_new, rr_cur, n, fp);
        CUR(cudaGetLastError());
        if ((st = hisq_push_end(h, s, p)) != DSLASH_OK) break;
        }
        if (!fused) CUR(cudaMemcpyAsync(&host_rr[k], rr_new, sizeof(double), cudaMemcpyDeviceToHost, s));
        CUR(cudaEventRecord(ev[k % (kCgLag + 1)], s));
        // check iteration k - kCgLag (complete or nearly) while the later ones run
        const int j = k - kCgLag;
        if (prof) {
            const double e = std::chrono::duration<double, std::micro>(clk::now() - t0).count();
            enq_us += e;
            enq_max = e > enq_max ? e : enq_max;
        }
        if (j >= 1) {
            const auto t1 = prof ? clk::now() : clk::time_point{};
            CUR(cudaEventSynchronize(ev[j % (kCgLag + 1)]));
            if (prof) wait_us += std::chrono::duration<double, std::micro>(clk::now() - t1).count();
            if (host_rr[j] <= stop) {
                kstar = j;
                break;
            }
        }
    }
    if (prof && k > 0)
        fprintf(stderr, "[hisq cg] %d iterations: enqueue %.1f us/iter (max %.1f), wait %.1f us/iter\n", k,
                enq_us / k, enq_max, wait_us / k);
    // the last direction update pushed faces of a p no apply will read
    if (st == DSLASH_OK) st = hisq_push_discard(h, s);
    if (st == DSLASH_OK) {
        if (k > max_iter) k = max_iter;
        CUR(cudaStreamSynchronize(s));
        if (!kstar)  // the last kCgLag iterations were not checked yet
            for (int j = k - kCgLag + 1 < 1 ? 1 : k - kCgLag + 1; j <= k; ++j)
                if (host_rr[j] <= stop) {
                    kstar = j;
                    break;
                }
        *converged = kstar > 0;
        if (kstar) k = kstar;
        *rr_last = host_rr[k];
    }
    *iters = k;
    release();
#undef CUR
    return st;
}

// |b - A x|^2 in fp64 (r receives the residual)
static dslash_status true_residual(dslash_t h, double2* r, const double2* x, const double2* b, int32_t parity,
                                   double m2, cudaStream_t s, double* rt) {
    const int64_t n = 3 * h->plan.vh_local;
    dslash_status st = normal_apply(h, r, x, parity, m2, (double2*)h->cg_vec[3], s, false);
    if (st != DSLASH_OK) return st;
    k_sub_from<<<kRedBlocks, kRedThreads, 0, s>>>(r, b, n);
    k_norm2<<<kRedBlocks, kRedThreads, 0, s>>>(r, n, h->cg_partial);
    CU(h, cudaGetLastError());
    return reduce_to_host(h, s, rt);
}

extern "C" dslash_status dslash_cg(dslash_t h, void* x_out, const void* b_in, int32_t parity, double mass,
                                   double rel_tol, int32_t max_iter, int32_t* iters, double* rel_resid,
                                   dslash_stream_t stream) {
    DeviceGuard device_guard(h);
    dslash_status st = check_solver_args(h, x_out, b_in, parity);
    if (st != DSLASH_OK) return st;
    if (!(rel_tol > 0.0) || max_iter < 1) return hisq_fail(h, DSLASH_ERR_ARG, "rel_tol must be > 0 and max_iter >= 1");
    if (!(mass != 0.0)) return hisq_fail(h, DSLASH_ERR_ARG, "mass must be nonzero (A is then positive definite)");
    if ((st = need_scratch(h)) != DSLASH_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t n = 3 * h->plan.vh_local;
    const size_t bytes = n * sizeof(double2);
    const double m2 = mass * mass;
    double2* x = (double2*)x_out;
    const double2* b = (const double2*)b_in;
    double2* r = (double2*)h->cg_vec[0];
    double2* p = (double2*)h->cg_vec[1];
    double2* q = (double2*)h->cg_vec[2];
    double2* t = (double2*)h->cg_vec[3];
    // x = 0, r = b, p = b
    CU(h, cudaMemsetAsync(x, 0, bytes, s));
    CU(h, cudaMemcpyAsync(r, b, bytes, cudaMemcpyDeviceToDevice, s));
    CU(h, cudaMemcpyAsync(p, b, bytes, cudaMemcpyDeviceToDevice, s));
    double bb = 0.0;
    k_norm2<<<kRedBlocks, kRedThreads, 0, s>>>(b, n, h->cg_partial);
    CU(h, cudaGetLastError());
    if ((st = reduce_to_host(h, s, &bb)) != DSLASH_OK) return st;
    int32_t k = 0;
    bool converged = !(bb > 0.0);
    double res = 0.0;
    if (bb > 0.0) {
        CU(h, cudaMemcpyAsync(&h->cg_scalar[0], &bb, sizeof(double), cudaMemcpyHostToDevice, s));
        double rr_last = 0.0;
        st = cg_core(h, x, r, p, q, t, parity, m2, rel_tol * rel_tol * bb, max_iter, s, &k, &rr_last, &converged);
        if (st != DSLASH_OK) return st;
        double rt = 0.0;  // true residual |b - A x| / |b|
        if ((st = true_residual(h, r, x, b, parity, m2, s, &rt)) != DSLASH_OK) return st;
        res = std::sqrt(rt / bb);
    }
    if (iters) *iters = k;
    if (rel_resid) *rel_resid = res;
    // not converged: reported, but not a sticky handle error
    return converged ? DSLASH_OK : DSLASH_ERR_NOT_CONVERGED;
}

// ---------------------------------------------------------------------------- mixed precision
// The fp32 ("sloppy") links of both parities, converted once from the handle's fp64 internal
// links into the fp32 paired layout the F32 kernels read (links.cuh convert_internal_kernel).
static dslash_status need_sloppy(dslash_t h) {
    const int64_t n = 3 * h->plan.vh_local;
    for (void*& v : h->cg_vec32)
        if (!v) CU(h, cudaMalloc(&v, n * sizeof(float2)));
    if (h->links32[0]) return DSLASH_OK;
    for (int par = 0; par < 2; ++par) {
        // fp32 paired links of the same recon (recon-9 links are stored in full: 144 entries)
        const size_t bytes32 = h->recon == 9 ? (size_t)h->plan.vh_local * 144 * sizeof(float2) : h->link_bytes / 2;
        CU(h, cudaMalloc(&h->links32[par], bytes32));
        dslash_status st = hisq_convert_links_sloppy(h, par);
        if (st != DSLASH_OK) return st;
    }
    return DSLASH_OK;
}

// Run the handle as an fp32 one (F32 kernels on the sloppy links) for the inner solve; every
// rank does the same, so halo messages keep matching sizes.
struct SloppyScope {
    dslash_t h;
    int precision, recon;
    void* links[2];
    explicit SloppyScope(dslash_t hh) : h(hh), precision(hh->precision), recon(hh->recon) {
        links[0] = h->links[0];
        links[1] = h->links[1];
        h->precision = DSLASH_F32;
        if (h->recon == 9) h->recon = 18;  // the fp32 copies of recon-9 links are stored in full
        h->links[0] = h->links32[0];
        h->links[1] = h->links32[1];
    }
    ~SloppyScope() {
        h->precision = precision;
        h->recon = recon;
        h->links[0] = links[0];
        h->links[1] = links[1];
    }
};

extern "C" dslash_status dslash_cg_mixed(dslash_t h, void* x_out, const void* b_in, int32_t parity, double mass,
                                         double rel_tol, double inner_tol, int32_t max_iter, int32_t* iters,
                                         int32_t* outer_iters, double* rel_resid, dslash_stream_t stream) {
    DeviceGuard device_guard(h);
    dslash_status st = check_solver_args(h, x_out, b_in, parity);
    if (st != DSLASH_OK) return st;
    if (h->precision != DSLASH_F64)
        return hisq_fail(h, DSLASH_ERR_UNSUPPORTED, "the mixed-precision solver needs an fp64 handle (DSLASH_F64)");
    if (!(rel_tol > 0.0) || max_iter < 1 || !(inner_tol > 0.0) || !(inner_tol < 1.0))
        return hisq_fail(h, DSLASH_ERR_ARG, "need rel_tol > 0, 0 < inner_tol < 1, max_iter >= 1");
    if (!(mass != 0.0)) return hisq_fail(h, DSLASH_ERR_ARG, "mass must be nonzero (A is then positive definite)");
    if ((st = need_scratch(h)) != DSLASH_OK) return st;
    if ((st = need_sloppy(h)) != DSLASH_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t n = 3 * h->plan.vh_local;
    const double m2 = mass * mass;
    double2* x = (double2*)x_out;
    const double2* b = (const double2*)b_in;
    double2* r = (double2*)h->cg_vec[0];
    float2* e = (float2*)h->cg_vec32[0];
    float2* r32 = (float2*)h->cg_vec32[1];
    float2* p32 = (float2*)h->cg_vec32[2];
    float2* q32 = (float2*)h->cg_vec32[3];
    float2* t32 = (float2*)h->cg_vec32[4];
    CU(h, cudaMemsetAsync(x, 0, n * sizeof(double2), s));
    CU(h, cudaMemcpyAsync(r, b, n * sizeof(double2), cudaMemcpyDeviceToDevice, s));
    double bb = 0.0;
    k_norm2<<<kRedBlocks, kRedThreads, 0, s>>>(b, n, h->cg_partial);
    CU(h, cudaGetLastError());
    if ((st = reduce_to_host(h, s, &bb)) != DSLASH_OK) return st;
    // Defect correction (iterative refinement): r = b - A x in fp64; solve A e = r in fp32 CG to
    // relative residual inner_tol; x += e in fp64; repeat until |r| <= rel_tol |b|.
    double rr = bb;
    int32_t total = 0, outer = 0;
    bool converged = !(bb > 0.0);
    while (!converged && total < max_iter) {
        if (rr <= rel_tol * rel_tol * bb) {
            converged = true;
            break;
        }
        k_round_to_f32<<<kRedBlocks, kRedThreads, 0, s>>>(r32, r, n);
        CU(h, cudaGetLastError());
        CU(h, cudaMemcpyAsync(p32, r32, n * sizeof(float2), cudaMemcpyDeviceToDevice, s));
        CU(h, cudaMemsetAsync(e, 0, n * sizeof(float2), s));
        double rr32 = 0.0;
        k_norm2<<<kRedBlocks, kRedThreads, 0, s>>>(r32, n, h->cg_partial);
        CU(h, cudaGetLastError());
        if ((st = reduce_to_slot(h, s, &h->cg_scalar[0])) != DSLASH_OK) return st;  // sc[0] = <r32, r32>
        CU(h, cudaMemcpyAsync(&rr32, &h->cg_scalar[0], sizeof(double), cudaMemcpyDeviceToHost, s));
        CU(h, cudaStreamSynchronize(s));
        int32_t k = 0;
        double rr_inner = 0.0;
        bool inner_conv = false;
        {
            SloppyScope scope(h);
            st = cg_core(h, e, r32, p32, q32, t32, parity, m2, inner_tol * inner_tol * rr32, max_iter - total, s, &k,
                         &rr_inner, &inner_conv);
        }
        if (st != DSLASH_OK) return st;
        total += k;
        ++outer;
        k_add_f32<<<kRedBlocks, kRedThreads, 0, s>>>(x, e, n);
        CU(h, cudaGetLastError());
        if ((st = true_residual(h, r, x, b, parity, m2, s, &rr)) != DSLASH_OK) return st;
    }
    if (!converged && rr <= rel_tol * rel_tol * bb) converged = true;
    if (iters) *iters = total;
    if (outer_iters) *outer_iters = outer;
    if (rel_resid) *rel_resid = bb > 0.0 ? std::sqrt(rr / bb) : 0.0;
    return converged ? DSLASH_OK : DSLASH_ERR_NOT_CONVERGED;
}
