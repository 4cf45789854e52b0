// kernels_rhs8.cu -- the TMA-fed 8-RHS kernel (rhs8_tma.cuh) and its launcher.
#include <cstdlib>

#include "dispatch.h"
#include "rhs8_tma.cuh"

namespace hisq {

template <int UNROLL, int NRHS>
static cudaError_t launch_t(const CUtensorMap& map, const StencilParams& P, int nsm, bool pdl, cudaStream_t s) {
    using C = Rhs8Cfg<NRHS>;
    auto fn = dslash_rhs8_tma_kernel<UNROLL, NRHS>;
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::smem());
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    const int64_t tiles = P.vh / C::TS;
    const int64_t blocks = (tiles + C::WARPS - 1) / C::WARPS;
    const unsigned grid = (unsigned)(blocks < C::MINB * (int64_t)nsm ? blocks : C::MINB * (int64_t)nsm);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(32 * C::WARPS);
    cfg.dynamicSmemBytes = C::smem();
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, fn, map, P);
}

int rhs8_tile_sites() {
    static const int nrhs = getenv("HISQ_RHS8_NRHS") ? atoi(getenv("HISQ_RHS8_NRHS")) : 4;
    return nrhs == 2 ? Rhs8Cfg<2>::TS : Rhs8Cfg<4>::TS;
}

cudaError_t launch_rhs8_tma(const CUtensorMap& map, const StencilParams& P, int nsm, bool pdl, cudaStream_t s) {
    // HISQ_RHS8_UNROLL / HISQ_RHS8_NRHS (measurement aids): hops unrolled per direction (4) or
    // rolled (1); 4 or 2 right-hand sides per thread
    static const int unroll = getenv("HISQ_RHS8_UNROLL") ? atoi(getenv("HISQ_RHS8_UNROLL")) : 1;
    static const int nrhs = getenv("HISQ_RHS8_NRHS") ? atoi(getenv("HISQ_RHS8_NRHS")) : 4;
    if (nrhs == 2) return unroll == 4 ? launch_t<4, 2>(map, P, nsm, pdl, s) : launch_t<1, 2>(map, P, nsm, pdl, s);
    return unroll == 4 ? launch_t<4, 4>(map, P, nsm, pdl, s) : launch_t<1, 4>(map, P, nsm, pdl, s);
}

}  // namespace hisq
