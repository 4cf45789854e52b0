// solver_multi.cu -- conjugate gradient for nrhs independent systems A_p x_r = b_r that share every
// pass over the links: SURVEY.md §8(f)-3 (the CG on the normal operator) run on the
// §8(f)-4 multi-RHS stencil (the L25 intensity argument), in the site-blocked vector layout of
// dslash_apply_multi_blocked.
//
// A_p = m^2 - D_{p,1-p} D_{1-p,p} (solver.cu).  Each right-hand side follows the Hestenes-Stiefel
// recurrences of dslash_cg on its own scalars (alpha_r, beta_r); only the two stencil applies per
// iteration are shared, as one 8-RHS launch each.  A system whose <r, r> reached its stopping value
// is frozen (alpha_r = 0) while the others continue; its iteration count is recorded on the device.
// Dot products: double-double sums over a fixed grid (deterministic), one rank.
#include <cmath>
#include <vector>

#include "common.cuh"
#include "handle.h"

namespace {

using hisq::dd_add;
using hisq::dot_term;

constexpr int kT = 256;          // threads per block
constexpr int kBlocksPerRhs = 148;
constexpr int kMaxRhs = 8;       // one stencil launch
constexpr int kCheckEvery = 8;   // iterations between host convergence checks

// complex element j (0 <= j < 3 Vh) of right-hand side r of a site-blocked vector of nrhs: the
// r-th 48 (3 colour rows of 16) of every 16-site block
__device__ __forceinline__ int64_t bidx(int64_t j, int r, int nrhs) {
    return (j / 48) * (48 * (int64_t)nrhs) + 48 * r + j % 48;
}

__device__ double2 block_sum_m(double2 v) {
    __shared__ double2 warp_part[kT / 32];
#pragma unroll
    for (int off = 16; off; off >>= 1)
        v = dd_add(v, make_double2(__shfl_xor_sync(0xffffffffu, v.x, off), __shfl_xor_sync(0xffffffffu, v.y, off)));
    if ((threadIdx.x & 31) == 0) warp_part[threadIdx.x >> 5] = v;
    __syncthreads();
    double2 s = make_double2(0.0, 0.0);
    if (threadIdx.x == 0)
        for (int w = 0; w < kT / 32; ++w) s = dd_add(s, warp_part[w]);
    return s;
}

// grid (kBlocksPerRhs, nrhs): blockIdx.y = right-hand side.  q = m2 p - q ; partial = Re<p, q>
__global__ void __launch_bounds__(kT) k_m_normal_finish(const double2* __restrict__ p, double2* __restrict__ q,
                                                        double m2, int nrhs, int64_t n, double2* __restrict__ partial) {
    const int r = blockIdx.y;
    double2 acc = make_double2(0.0, 0.0);
    for (int64_t j = (int64_t)blockIdx.x * kT + threadIdx.x; j < n; j += (int64_t)gridDim.x * kT) {
        const int64_t i = bidx(j, r, nrhs);
        const double2 a = p[i];
        double2 b = q[i];
        b.x = m2 * a.x - b.x;
        b.y = m2 * a.y - b.y;
        q[i] = b;
        acc = dd_add(acc, dot_term(a, b));
    }
    const double2 s = block_sum_m(acc);
    if (threadIdx.x == 0) partial[r * kBlocksPerRhs + blockIdx.x] = s;
}

// partial = |v_r|^2
__global__ void __launch_bounds__(kT) k_m_norm2(const double2* __restrict__ v, int nrhs, int64_t n,
                                                double2* __restrict__ partial) {
    const int r = blockIdx.y;
    double2 acc = make_double2(0.0, 0.0);
    for (int64_t j = (int64_t)blockIdx.x * kT + threadIdx.x; j < n; j += (int64_t)gridDim.x * kT) {
        const double2 a = v[bidx(j, r, nrhs)];
        acc = dd_add(acc, dot_term(a, a));
    }
    const double2 s = block_sum_m(acc);
    if (threadIdx.x == 0) partial[r * kBlocksPerRhs + blockIdx.x] = s;
}

// one block per right-hand side: out[r] = the rounded double-double sum of its partials; with conv:
// the first iteration whose <r, r> (out) is <= stop[r] is recorded in conv[r]
__global__ void __launch_bounds__(kT) k_m_finalize(const double2* __restrict__ partial, double* __restrict__ out,
                                                   const double* __restrict__ stop, int* __restrict__ conv, int it) {
    const int r = blockIdx.x;
    double2 acc = make_double2(0.0, 0.0);
    for (int k = threadIdx.x; k < kBlocksPerRhs; k += kT) acc = dd_add(acc, partial[r * kBlocksPerRhs + k]);
    const double2 s = block_sum_m(acc);
    if (threadIdx.x == 0) {
        out[r] = s.x;
        if (conv && conv[r] < 0 && s.x <= stop[r]) conv[r] = it;
    }
}

// x_r += alpha_r p_r ; r_r -= alpha_r q_r ; partial = |r_r|^2, alpha_r = rr_r / pq_r (0 once frozen)
__global__ void __launch_bounds__(kT) k_m_update(double2* __restrict__ x, double2* __restrict__ res,
                                                 const double2* __restrict__ p, const double2* __restrict__ q,
                                                 const double* __restrict__ rr, const double* __restrict__ pq,
                                                 const double* __restrict__ stop, int nrhs, int64_t n,
                                                 double2* __restrict__ partial) {
    const int r = blockIdx.y;
    // a frozen system keeps x_r and r_r (its p_r is not updated either: no inf * 0)
    const bool frozen = !(rr[r] > stop[r]) || pq[r] == 0.0;
    const double alpha = frozen ? 0.0 : rr[r] / pq[r];
    double2 acc = make_double2(0.0, 0.0);
    for (int64_t j = (int64_t)blockIdx.x * kT + threadIdx.x; j < n; j += (int64_t)gridDim.x * kT) {
        const int64_t i = bidx(j, r, nrhs);
        if (frozen) {
            const double2 ri = res[i];
            acc = dd_add(acc, dot_term(ri, ri));
            continue;
        }
        double2 xi = x[i], ri = res[i];
        const double2 pi = p[i], qi = q[i];
        xi.x = fma(alpha, pi.x, xi.x);
        xi.y = fma(alpha, pi.y, xi.y);
        ri.x = fma(-alpha, qi.x, ri.x);
        ri.y = fma(-alpha, qi.y, ri.y);
        x[i] = xi;
        res[i] = ri;
        acc = dd_add(acc, dot_term(ri, ri));
    }
    const double2 s = block_sum_m(acc);
    if (threadIdx.x == 0) partial[r * kBlocksPerRhs + blockIdx.x] = s;
}

// p_r = r_r + beta_r p_r, beta_r = rr_new_r / rr_r; frozen systems (rr_r <= stop_r) keep p_r
__global__ void __launch_bounds__(kT) k_m_direction(double2* __restrict__ p, const double2* __restrict__ res,
                                                    const double* __restrict__ rr_new, const double* __restrict__ rr,
                                                    const double* __restrict__ stop, int nrhs, int64_t n) {
    const int r = blockIdx.y;
    if (!(rr[r] > stop[r])) return;
    const double beta = rr_new[r] / rr[r];
    for (int64_t j = (int64_t)blockIdx.x * kT + threadIdx.x; j < n; j += (int64_t)gridDim.x * kT) {
        const int64_t i = bidx(j, r, nrhs);
        const double2 ri = res[i];
        double2 pi = p[i];
        pi.x = fma(beta, pi.x, ri.x);
        pi.y = fma(beta, pi.y, ri.y);
        p[i] = pi;
    }
}

// res = b - res (elementwise, layout-free)
__global__ void k_m_sub_from(double2* __restrict__ res, const double2* __restrict__ b, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const double2 bi = b[i], ri = res[i];
        res[i] = make_double2(bi.x - ri.x, bi.y - ri.y);
    }
}

}  // namespace

extern "C" dslash_status dslash_cg_multi_blocked(dslash_t h, int32_t nrhs, void* x_out, const void* b_in,
                                                 int32_t parity, double mass, double rel_tol, int32_t max_iter,
                                                 int32_t* iters, double* rel_resid, dslash_stream_t stream) {
    DeviceGuard device_guard(h);
    if (!h) return hisq_fail(nullptr, DSLASH_ERR_ARG, "NULL handle");
    if (parity & ~1) return hisq_fail(h, DSLASH_ERR_ARG, "parity %d not in {0,1}", parity);
    if (nrhs < 1 || nrhs > kMaxRhs) return hisq_fail(h, DSLASH_ERR_ARG, "nrhs %d not in [1, %d]", nrhs, kMaxRhs);
    if (h->parity_mask != DSLASH_BOTH)
        return hisq_fail(h, DSLASH_ERR_ARG, "the normal operator applies both parities: create with DSLASH_BOTH");
    if (h->precision == DSLASH_F32)
        return hisq_fail(h, DSLASH_ERR_UNSUPPORTED, "the solver works on fp64 vectors (DSLASH_F64 or DSLASH_MIXED)");
    if (!h->loaded) return hisq_fail(h, DSLASH_ERR_STATE, "solver before load_links");
    if (h->plan.nranks > 1)
        return hisq_fail(h, DSLASH_ERR_UNSUPPORTED, "the multi-RHS solver runs on one rank (use dslash_cg per RHS)");
    if (!(rel_tol > 0.0) || max_iter < 1) return hisq_fail(h, DSLASH_ERR_ARG, "rel_tol must be > 0 and max_iter >= 1");
    if (!(mass != 0.0)) return hisq_fail(h, DSLASH_ERR_ARG, "mass must be nonzero (A is then positive definite)");
    const int64_t nper = 3 * h->plan.vh_local;  // complex per right-hand side
    const int64_t n = nper * nrhs;
    const size_t bytes = (size_t)n * sizeof(double2);
    if (!x_out || !b_in || ((uintptr_t)x_out & 15) || ((uintptr_t)b_in & 15))
        return hisq_fail(h, DSLASH_ERR_ARG, "NULL or misaligned vector");
    if ((uintptr_t)x_out < (uintptr_t)b_in + bytes && (uintptr_t)b_in < (uintptr_t)x_out + bytes)
        return hisq_fail(h, DSLASH_ERR_ARG, "vectors overlap");
    cudaStream_t s = (cudaStream_t)stream;
    const double m2 = mass * mass;
    // scratch kept on the handle (freed by dslash_destroy), grown when a larger solve needs it
    if (h->cgm_bytes < bytes) {
        for (void*& v : h->cgm_vec) {
            if (v) cudaFree(v);
            v = nullptr;
        }
        h->cgm_bytes = 0;
        for (void*& v : h->cgm_vec) CU(h, cudaMalloc(&v, bytes));
        h->cgm_bytes = bytes;
    }
    const size_t small = (size_t)kMaxRhs * kBlocksPerRhs * sizeof(double2) + 6 * kMaxRhs * sizeof(double) +
                         kMaxRhs * sizeof(int);
    if (!h->cgm_small) CU(h, cudaMalloc(&h->cgm_small, small));
    double2* r = static_cast<double2*>(h->cgm_vec[0]);
    double2* p = static_cast<double2*>(h->cgm_vec[1]);
    double2* q = static_cast<double2*>(h->cgm_vec[2]);
    double2* t = static_cast<double2*>(h->cgm_vec[3]);
    double2* partial = static_cast<double2*>(h->cgm_small);
    double* sc = reinterpret_cast<double*>(partial + kMaxRhs * kBlocksPerRhs);  // rr[2][nrhs], pq, stop, b2, tr
    int* conv = reinterpret_cast<int*>(sc + 6 * kMaxRhs);
    dslash_status st;
    double *rr0 = sc, *rr1 = sc + kMaxRhs, *pq = sc + 2 * kMaxRhs, *stop = sc + 3 * kMaxRhs, *b2 = sc + 4 * kMaxRhs,
           *tr = sc + 5 * kMaxRhs;
    double2* x = static_cast<double2*>(x_out);
    const double2* b = static_cast<const double2*>(b_in);
    const dim3 grid(kBlocksPerRhs, nrhs);
    // x = 0, r = p = b; <b_r, b_r> -> rr0 and b2; stop_r = tol^2 <b_r, b_r>
    CU(h, cudaMemsetAsync(x, 0, bytes, s));
    CU(h, cudaMemcpyAsync(r, b, bytes, cudaMemcpyDeviceToDevice, s));
    CU(h, cudaMemcpyAsync(p, b, bytes, cudaMemcpyDeviceToDevice, s));
    CU(h, cudaMemsetAsync(conv, 0xff, kMaxRhs * sizeof(int), s));  // -1: not converged
    k_m_norm2<<<grid, kT, 0, s>>>(b, nrhs, nper, partial);
    k_m_finalize<<<nrhs, kT, 0, s>>>(partial, rr0, nullptr, nullptr, 0);
    CU(h, cudaGetLastError());
    std::vector<double> hb2(nrhs), hstop(nrhs);
    CU(h, cudaMemcpyAsync(hb2.data(), rr0, nrhs * sizeof(double), cudaMemcpyDeviceToHost, s));
    CU(h, cudaStreamSynchronize(s));
    for (int k = 0; k < nrhs; ++k) hstop[k] = rel_tol * rel_tol * hb2[k];
    CU(h, cudaMemcpyAsync(b2, hb2.data(), nrhs * sizeof(double), cudaMemcpyHostToDevice, s));
    CU(h, cudaMemcpyAsync(stop, hstop.data(), nrhs * sizeof(double), cudaMemcpyHostToDevice, s));
    // systems with b_r = 0 are solved by x_r = 0 at iteration 0
    std::vector<int> hconv(nrhs, -1);
    for (int k = 0; k < nrhs; ++k)
        if (!(hb2[k] > 0.0)) hconv[k] = 0;
    CU(h, cudaMemcpyAsync(conv, hconv.data(), nrhs * sizeof(int), cudaMemcpyHostToDevice, s));
    double *rr = rr0, *rr_new = rr1;
    int it = 0;
    bool all = false;
    for (int k = 0; k < nrhs; ++k) all = all || hconv[k] < 0;
    all = !all;
    while (!all && it < max_iter) {
        ++it;
        // q = A p: two stencil passes over all nrhs systems, then q = m^2 p - q and <p, q>
        if ((st = hisq_apply_blocked(h, t, p, 1 - parity, nrhs, s)) != DSLASH_OK) return st;
        if ((st = hisq_apply_blocked(h, q, t, parity, nrhs, s)) != DSLASH_OK) return st;
        k_m_normal_finish<<<grid, kT, 0, s>>>(p, q, m2, nrhs, nper, partial);
        k_m_finalize<<<nrhs, kT, 0, s>>>(partial, pq, nullptr, nullptr, it);
        k_m_update<<<grid, kT, 0, s>>>(x, r, p, q, rr, pq, stop, nrhs, nper, partial);
        k_m_finalize<<<nrhs, kT, 0, s>>>(partial, rr_new, stop, conv, it);
        k_m_direction<<<grid, kT, 0, s>>>(p, r, rr_new, rr, stop, nrhs, nper);
        CU(h, cudaGetLastError());
        std::swap(rr, rr_new);
        if (it % kCheckEvery == 0 || it == max_iter) {
            CU(h, cudaMemcpyAsync(hconv.data(), conv, nrhs * sizeof(int), cudaMemcpyDeviceToHost, s));
            CU(h, cudaStreamSynchronize(s));
            all = true;
            for (int k = 0; k < nrhs; ++k) all = all && hconv[k] >= 0;
        }
    }
    CU(h, cudaMemcpyAsync(hconv.data(), conv, nrhs * sizeof(int), cudaMemcpyDeviceToHost, s));
    // true residuals |b_r - A x_r| / |b_r| in fp64
    if ((st = hisq_apply_blocked(h, t, x, 1 - parity, nrhs, s)) != DSLASH_OK) return st;
    if ((st = hisq_apply_blocked(h, r, t, parity, nrhs, s)) != DSLASH_OK) return st;
    k_m_normal_finish<<<grid, kT, 0, s>>>(x, r, m2, nrhs, nper, partial);  // r = A x (its <x, Ax> unused)
    k_m_sub_from<<<kBlocksPerRhs * 4, kT, 0, s>>>(r, b, n);
    k_m_norm2<<<grid, kT, 0, s>>>(r, nrhs, nper, partial);
    k_m_finalize<<<nrhs, kT, 0, s>>>(partial, tr, nullptr, nullptr, 0);
    CU(h, cudaGetLastError());
    std::vector<double> htr(nrhs);
    CU(h, cudaMemcpyAsync(htr.data(), tr, nrhs * sizeof(double), cudaMemcpyDeviceToHost, s));
    CU(h, cudaStreamSynchronize(s));
    bool converged = true;
    for (int k = 0; k < nrhs; ++k) {
        converged = converged && hconv[k] >= 0;
        if (iters) iters[k] = hconv[k] >= 0 ? hconv[k] : it;
        if (rel_resid) rel_resid[k] = hb2[k] > 0.0 ? std::sqrt(htr[k] / hb2[k]) : 0.0;
    }
    return converged ? DSLASH_OK : DSLASH_ERR_NOT_CONVERGED;
}
