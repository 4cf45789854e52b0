// kernels_rhs8.cu -- the TMA-fed 8-RHS kernel (rhs8_tma.cuh) and its launcher.
#include <cstdlib>

#include "dispatch.h"
#include "rhs8_tma.cuh"

namespace hisq {

cudaError_t launch_rhs8_tma(const CUtensorMap& map, const StencilParams& P, int nsm, bool pdl, cudaStream_t s) {
    // HISQ_RHS8_UNROLL (measurement aid): hops unrolled per direction (4) or rolled (1)
    static const int unroll = getenv("HISQ_RHS8_UNROLL") ? atoi(getenv("HISQ_RHS8_UNROLL")) : 1;
    void (*fn)(const CUtensorMap, const StencilParams) =
        unroll == 4 ? dslash_rhs8_tma_kernel<4> : dslash_rhs8_tma_kernel<1>;
    static bool attr_set[2] = {false, false};
    const size_t smem = rhs8_smem_bytes();
    if (!attr_set[unroll == 4]) {
        cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr_set[unroll == 4] = true;
    }
    const int64_t tiles = P.vh / kRhs8Sites;
    const int64_t blocks = (tiles + kRhs8Warps - 1) / kRhs8Warps;
    const unsigned grid = (unsigned)(blocks < 2 * (int64_t)nsm ? blocks : 2 * (int64_t)nsm);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(32 * kRhs8Warps);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, fn, map, P);
}

}  // namespace hisq
