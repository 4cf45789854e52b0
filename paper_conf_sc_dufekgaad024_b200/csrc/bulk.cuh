// bulk.cuh -- the TMA-staged Dslash kernel (DSLASH_KERNEL_BULK): a persistent, warp-specialised
// producer/consumer pipeline that streams link tiles into shared memory with cp.async.bulk
// (the Blackwell TMA engine, SASS UBLKCP) and mbarrier completion, instead of per-thread loads.
//
// Why: the register-staged kernels keep at most ~2 link matrices per thread in
// flight.  Here the TMA engine keeps 2 tiles (2 x 18 KB) per warp in flight regardless of
// register pressure, and the persistent grid (one CTA per SM) takes tiles from a global atomic
// counter in lattice (t-slowest) order, so all SMs sweep the lattice together and every SM stays
// busy until the tile pool is empty.
//
// Tile = 8 consecutive target sites of one x-row.  The tiled link layout keeps a tile's 16
// matrices contiguous:  links[(tile * E + base(l) + e) * 32 + s * 4 + mu],  tile = cb / 8,
// s = cb % 8, E = 36 (30 with recon-12), so one bulk copy moves a whole tile.  In a warp,
// lane = (site s, direction mu): the DIR4 mapping with a 2-step __shfl_xor butterfly.  The 12
// neighbour-vector loads of a tile are issued before waiting for its links.
#pragma once

#include "common.cuh"
#include "stencil.cuh"

namespace hisq {

constexpr int kBulkTile = 8;   // target sites per tile (lxh must be a multiple)
constexpr int kBulkWarps = 6;  // warps per CTA, each with 2 stages of 18 KB (fp64): 221 KB of smem
constexpr int kBulkBatch = 4;  // tiles per ticket draw

template <int RECON>
__host__ __device__ constexpr int bulk_elems() { return RECON == 12 ? 30 : 36; }

template <int RECON>
__host__ __device__ __forceinline__ int64_t link_index_tiled(int mu, int l, int e, int64_t cb) {
    return ((cb / kBulkTile) * bulk_elems<RECON>() + elem_base<RECON>(l) + e) * (kBulkTile * 4) +
           (cb % kBulkTile) * 4 + mu;
}

// ---------------------------------------------------------------- the kernel
// Every warp is its own producer: lane 0 draws tiles from a global ticket counter (zeroed before
// the launch) in batches, broadcasts them with __shfl_sync and keeps two bulk copies in flight
// into the warp's own two stages, so the next tile's links stream while the current one is
// computed.  The mbarriers carry only TMA transaction completion, and no thread reads shared
// memory written by another warp (compute-sanitizer racecheck: 0 hazards).
template <typename LR, typename VR, bool GHOST, int RECON>
__global__ void __launch_bounds__(32 * kBulkWarps, 1)
    dslash_bulk_kernel(const StencilParams P, unsigned long long* sched, unsigned long long /*unused*/) {
    using L2 = cplx_t<LR>;
    using V2 = cplx_t<VR>;
    constexpr int E = bulk_elems<RECON>();
    constexpr uint32_t kTileBytes = (uint32_t)(E * kBulkTile * 4 * sizeof(L2));
    extern __shared__ __align__(128) unsigned char smem[];
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    L2* my_stage[2] = {reinterpret_cast<L2*>(smem + (size_t)(2 * warp) * kTileBytes),
                       reinterpret_cast<L2*>(smem + (size_t)(2 * warp + 1) * kTileBytes)};
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + (size_t)2 * kBulkWarps * kTileBytes) + 2 * warp;
    const long long ntiles = (long long)(P.box_start[P.nbox] / kBulkTile);
    const uint64_t pol = policy_evict_first();
    const uint64_t pol_keep = policy_evict_last();
    const unsigned char* links = static_cast<const unsigned char*>(P.links);

    if (lane == 0) {
        mbar_init(&full[0], 1);
        mbar_init(&full[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    // lane 0: tickets in batches of kBulkBatch (the counter was zeroed before the launch), the next
    // batch always in flight; tiles past the pool come back as ntiles
    long long bcur = 0, bnext = 0;
    int icur = 0;
    if (lane == 0) {
        bcur = (long long)atomicAdd(sched, (unsigned long long)kBulkBatch);
        bnext = (long long)atomicAdd(sched, (unsigned long long)kBulkBatch);
    }
    auto next_tile = [&]() -> long long {  // lane 0 only
        if (icur == kBulkBatch) {
            bcur = bnext;
            icur = 0;
            if (bcur < ntiles) bnext = (long long)atomicAdd(sched, (unsigned long long)kBulkBatch);
        }
        const long long t = bcur + icur++;
        return t < ntiles ? t : ntiles;
    };
    auto issue = [&](int slot, long long tile) {  // lane 0 only
        const Site s0 = decode_site(P, tile * kBulkTile);
        mbar_arrive_expect_tx(&full[slot], kTileBytes);
        bulk_g2s(my_stage[slot], links + (size_t)(s0.cb / kBulkTile) * kTileBytes, kTileBytes, &full[slot], pol);
    };
    long long t_cur = 0, t_nxt = 0;
    if (lane == 0) {
        t_cur = next_tile();
        if (t_cur < ntiles) issue(0, t_cur);
        t_nxt = next_tile();
        if (t_nxt < ntiles) issue(1, t_nxt);
    }
    t_cur = __shfl_sync(0xffffffffu, t_cur, 0);
    t_nxt = __shfl_sync(0xffffffffu, t_nxt, 0);
    const int s_in_tile = lane >> 2;
    const int mu = lane & 3;
    uint32_t phase[2] = {0u, 0u};
    for (int it = 0; t_cur < ntiles; ++it) {
        const int slot = it & 1;
        long long t_after = 0;
        if (lane == 0) t_after = next_tile();
        const Site s = decode_site(P, t_cur * kBulkTile + s_in_tile);
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
        mbar_wait(&full[slot], phase[slot]);
        phase[slot] ^= 1u;
        const L2* stage = my_stage[slot];
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
        __syncwarp();  // every lane has read the stage: it may be refilled
        if (lane == 0 && t_after < ntiles) issue(slot, t_after);
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
        t_cur = t_nxt;
        t_nxt = __shfl_sync(0xffffffffu, t_after, 0);
    }
}

template <typename LR, int RECON>
constexpr size_t bulk_smem_bytes() {
    return (size_t)2 * kBulkWarps * bulk_elems<RECON>() * kBulkTile * 4 * sizeof(cplx_t<LR>) +
           2 * kBulkWarps * sizeof(uint64_t);  // two stages and two full barriers per warp
}

}  // namespace hisq
