// bulk.cuh -- the TMA-staged Dslash kernel (DSLASH_KERNEL_BULK): a persistent, warp-specialised
// producer/consumer pipeline that streams link tiles into shared memory with cp.async.bulk
// (the Blackwell TMA engine, SASS UBLKCP) and mbarrier completion, instead of per-thread loads.
//
// Why: the register-staged kernels keep at most ~2 link matrices per thread in
// flight and lose ~5% at 32^4 to the launch's ramp and tail.  Here one elected thread per CTA
// keeps S tiles (S x 18 KB) in flight regardless of register pressure, and the persistent grid
// (one CTA per SM) takes tiles from a global atomic counter in lattice (t-slowest) order, so
// all SMs sweep the lattice together and every SM stays busy until the tile pool is empty.
//
// Tile = 8 consecutive target sites of one x-row.  The tiled link layout keeps a tile's 16
// matrices contiguous:  links[(tile * E + base(l) + e) * 32 + s * 4 + mu],  tile = cb / 8,
// s = cb % 8, E = 36 (30 with recon-12), so one bulk copy moves a whole tile.  A consumer warp
// computes the CTA's k-th tile for k = w, w + W, ... from stage k mod S (S = W): the producer
// publishes the tile index next to the stage; lane = (site s, direction mu), the DIR4 mapping
// with a 2-step __shfl_xor butterfly.  The 12 neighbour-vector loads are issued right after the
// tile index is known, before the links are read, so the L2 gather latency overlaps the FMAs
// of the previous tile of the other warps.
#pragma once

#include "common.cuh"
#include "stencil.cuh"

namespace hisq {

constexpr int kBulkTile = 8;       // target sites per tile (lxh must be a multiple)
constexpr int kBulkConsumers = 8;  // consumer warps per CTA
constexpr int kBulkStages = 8;     // stage ring depth: one stage per consumer warp
constexpr int kBulkBatch = 4;      // tiles per scheduler ticket draw

template <int RECON>
__host__ __device__ constexpr int bulk_elems() { return RECON == 12 ? 30 : 36; }

template <int RECON>
__host__ __device__ __forceinline__ int64_t link_index_tiled(int mu, int l, int e, int64_t cb) {
    return ((cb / kBulkTile) * bulk_elems<RECON>() + elem_base<RECON>(l) + e) * (kBulkTile * 4) +
           (cb % kBulkTile) * 4 + mu;
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

// ---------------------------------------------------------------- the kernel
// sched: a 64-bit counter shared by the launches of one handle.  A producer draws batches of
// kBulkBatch tiles and always has the next draw in flight (its latency overlaps the current
// batch); it stops at the first batch past the pool, so every CTA makes exactly 2 draws that
// process nothing and a launch consumes (ceil(ntiles / B) + 2 gridDim.x) * B tickets, starting
// at sched_base.
template <typename LR, typename VR, bool GHOST, int RECON>
__global__ void __launch_bounds__(32 * (kBulkConsumers + 1), 1)
    dslash_bulk_kernel(const StencilParams P, unsigned long long* sched, unsigned long long sched_base) {
    using L2 = cplx_t<LR>;
    using V2 = cplx_t<VR>;
    constexpr int E = bulk_elems<RECON>();
    constexpr uint32_t kTileBytes = (uint32_t)(E * kBulkTile * 4 * sizeof(L2));
    extern __shared__ __align__(128) unsigned char smem[];
    L2* stage_base = reinterpret_cast<L2*>(smem);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + kBulkStages * kTileBytes);
    uint64_t* empty = full + kBulkStages;
    volatile long long* tile_of = reinterpret_cast<volatile long long*>(empty + kBulkStages);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const long long ntiles = (long long)(P.box_start[P.nbox] / kBulkTile);

    if (threadIdx.x == 0) {
        for (int i = 0; i < kBulkStages; ++i) {
            mbar_init(&full[i], 1);
            mbar_init(&empty[i], 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    if (warp == kBulkConsumers) {
        // ---------------- producer: one elected lane draws tiles and streams them into the ring
        if (lane == 0) {
            const uint64_t pol = policy_evict_first();
            const unsigned char* links = static_cast<const unsigned char*>(P.links);
            long long k = 0;
            long long batch = (long long)(atomicAdd(sched, (unsigned long long)kBulkBatch) - sched_base);
            for (;;) {
                const long long next = (long long)(atomicAdd(sched, (unsigned long long)kBulkBatch) - sched_base);
                if (batch >= ntiles) break;
                const long long end = batch + kBulkBatch < ntiles ? batch + kBulkBatch : ntiles;
                for (long long tile = batch; tile < end; ++tile, ++k) {
                    const int st = (int)(k % kBulkStages);
                    const uint32_t phase = (uint32_t)(k / kBulkStages) & 1u;
                    mbar_wait(&empty[st], phase ^ 1u);  // fresh barrier: passes immediately
                    tile_of[st] = tile;
                    // tile index in the box enumeration -> checkerboard tile (boxes hold whole x-rows)
                    const Site s0 = decode_site(P, tile * kBulkTile);
                    mbar_arrive_expect_tx(&full[st], kTileBytes);  // release: publishes tile_of[st]
                    bulk_g2s(stage_base + (size_t)st * (kTileBytes / sizeof(L2)),
                             links + (size_t)(s0.cb / kBulkTile) * kTileBytes, kTileBytes, &full[st], pol);
                }
                batch = next;
            }
            // stop every consumer: a sentinel in the next stage of each warp
            for (int j = 0; j < kBulkStages; ++j, ++k) {
                const int st = (int)(k % kBulkStages);
                const uint32_t phase = (uint32_t)(k / kBulkStages) & 1u;
                mbar_wait(&empty[st], phase ^ 1u);
                tile_of[st] = -1;
                mbar_arrive(&full[st]);
            }
        }
        return;
    }

    // ---------------- consumers: warp w computes the CTA's tiles k = w, w + W, ... from stage k mod S
    const int s_in_tile = lane >> 2;
    const int mu = lane & 3;
    const uint64_t pol_keep = policy_evict_last();
    for (long long k = warp;; k += kBulkConsumers) {
        const int st = (int)(k % kBulkStages);
        const uint32_t phase = (uint32_t)(k / kBulkStages) & 1u;
        mbar_wait(&full[st], phase);  // the tile index is published; the links may still be landing
        const long long tile = tile_of[st];
        if (tile < 0) break;
        const L2* stage = stage_base + (size_t)st * (kTileBytes / sizeof(L2));
        const Site s = decode_site(P, tile * kBulkTile + s_in_tile);
        V2 v[4][3];
#pragma unroll
        for (int l = 0; l < 4; ++l) {
            const int h = (l == 0) ? 1 : (l == 1) ? -1 : (l == 2) ? 3 : -3;
            const SrcRef<V2> src = source<V2, GHOST>(P, P.in, mu, h, s, 0);
#pragma unroll
            for (int c = 0; c < 3; ++c) v[l][c] = ld_reuse(src.p + c * src.stride, pol_keep);
        }
        V2 acc[3];
#pragma unroll
        for (int c = 0; c < 3; ++c) acc[c].x = acc[c].y = VR(0);
#pragma unroll
        for (int l = 0; l < 4; ++l) {
            V2 U[9];
#pragma unroll
            for (int e = 0; e < elems_of<RECON>(l); ++e)
                U[e] = to_cplx<V2>(widen(lds(stage + (elem_base<RECON>(l) + e) * (kBulkTile * 4) + lane)));
            if (elems_of<RECON>(l) == 6) reconstruct_row2(U, (VR)P.long_inv_scale);
            if (l & 1)
                matvec_acc<true>(acc, U, v[l]);
            else
                matvec_acc<false>(acc, U, v[l]);
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[st]);  // stage free for the producer
#pragma unroll
        for (int c = 0; c < 3; ++c) {
#pragma unroll
            for (int off = 1; off <= 2; off <<= 1) {
                acc[c].x += __shfl_xor_sync(0xffffffffu, acc[c].x, off);
                acc[c].y += __shfl_xor_sync(0xffffffffu, acc[c].y, off);
            }
        }
        if (mu < 3) {
            V2* out = static_cast<V2*>(P.out);
            st_stream(out + mu * P.vh + s.cb, mu == 0 ? acc[0] : mu == 1 ? acc[1] : acc[2]);
        }
    }
}

template <typename LR, int RECON>
constexpr size_t bulk_smem_bytes() {
    return (size_t)kBulkStages * bulk_elems<RECON>() * kBulkTile * 4 * sizeof(cplx_t<LR>) +
           3 * kBulkStages * sizeof(uint64_t);  // full, empty barriers and the published tile indices
}

}  // namespace hisq
