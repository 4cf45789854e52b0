// kernels_bulk.cu -- instantiations of the TMA-staged kernel (bulk.cuh) and its launch helper.
#include "bulk.cuh"
#include "dispatch.h"

namespace hisq {

template <typename LR, typename VR, int RECON>
static BulkKernel pick_bulk_t(bool ghost) {
    BulkKernel k;
    k.fn = ghost ? dslash_bulk_kernel<LR, VR, true, RECON> : dslash_bulk_kernel<LR, VR, false, RECON>;
    k.smem = bulk_smem_bytes<LR, RECON>();
    k.threads = 32 * kBulkWarps;
    k.tile = kBulkTile;
    k.batch = 1;
    // opt in to > 48 KB of dynamic shared memory (idempotent)
    cudaFuncSetAttribute(k.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)k.smem);
    return k;
}

BulkKernel pick_bulk(int precision, int recon, bool ghost) {
    const bool r12 = recon == 12;
    switch (precision) {
        case 1: return r12 ? pick_bulk_t<float, float, 12>(ghost) : pick_bulk_t<float, float, 18>(ghost);
        case 2: return r12 ? pick_bulk_t<float, double, 12>(ghost) : pick_bulk_t<float, double, 18>(ghost);
        default: return r12 ? pick_bulk_t<double, double, 12>(ghost) : pick_bulk_t<double, double, 18>(ghost);
    }
}

}  // namespace hisq
