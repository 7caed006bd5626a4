// st27t_inst.cu — instantiates the 27-point sweep on the 7-point machinery
// (st27t_kernel.cuh, tolerance build) for FP32 / FP64.
#include "launch.h"
#include "st27t_kernel.cuh"

namespace st35d {
namespace {

template <typename T, int D, int VY>
cudaError_t launch27t(const CUtensorMap* map, const St27tParams& p, int grid, int threads, size_t smem,
                      cudaStream_t s) {
    constexpr int NTX = sizeof(T) == 4 ? 16 : 32;
    auto k = st27t_kernel<T, D, NTX, VY, 256>;
    if (threads > 256 || threads % NTX) return cudaErrorInvalidValue;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return launch_pdl(p.g.pdl != 0, k, grid, threads, smem, s, *map, p);
}

template <typename T>
St27tLaunchFn pick27t(int D, int VY) {
    if (VY == 4) {
        switch (D) {
            case 1: return launch27t<T, 1, 4>;
            case 2: return launch27t<T, 2, 4>;
            default: return nullptr;
        }
    }
    if (VY == 2) {
        switch (D) {
            case 1: return launch27t<T, 1, 2>;
            case 2: return launch27t<T, 2, 2>;
            case 3: return launch27t<T, 3, 2>;
            case 4: return launch27t<T, 4, 2>;
            default: return nullptr;
        }
    }
    return nullptr;
}

}  // namespace

// compiled variants: VY = 4 rows per thread (dim_T <= 2), VY = 2 (dim_T <= 4); 256 threads max
St27tLaunchFn st27t_lookup(int dtype, int D, int VY) {
    return dtype == 0 ? pick27t<float>(D, VY) : pick27t<double>(D, VY);
}

}  // namespace st35d
