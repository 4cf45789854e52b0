// kernels_rhs8.cu -- the TMA-fed 8-RHS kernel (rhs8_tma.cuh) and its launcher.
#include "dispatch.h"
#include "rhs8_tma.cuh"

namespace hisq {

cudaError_t launch_rhs8_tma(const CUtensorMap& map, const StencilParams& P, int nsm, bool pdl, cudaStream_t s) {
    static bool attr_set = false;
    const size_t smem = rhs8_smem_bytes();
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(dslash_rhs8_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr_set = true;
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
    return cudaLaunchKernelEx(&cfg, dslash_rhs8_tma_kernel, map, P);
}

}  // namespace hisq
