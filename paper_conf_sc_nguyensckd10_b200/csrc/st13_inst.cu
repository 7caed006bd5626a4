// st13_inst.cu — instantiates the radius-2 sweep kernel (st13_kernel.cuh) for
// FP32/FP64 in the tolerance and bit-exact builds.
#include "launch.h"
#include "st13_kernel.cuh"

namespace st35d {
namespace {

template <typename T, int D, int VY, bool E>
cudaError_t launch13(const CUtensorMap* map, const St13Params& p, int grid, int threads, size_t smem, cudaStream_t s) {
    constexpr int NTX = sizeof(T) == 4 ? 16 : 32;
    auto k = st13_35d_kernel<T, D, NTX, VY, E, 256>;
    if (threads > 256 || threads % NTX) return cudaErrorInvalidValue;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return launch_pdl(p.g.pdl != 0, k, grid, threads, smem, s, *map, p);
}

template <typename T, bool E>
St13LaunchFn pick13(int D, int VY) {
    if (VY == 4) {
        switch (D) {
            case 1: return launch13<T, 1, 4, E>;
            case 2: return launch13<T, 2, 4, E>;
            default: return nullptr;
        }
    }
    if (VY == 2) {
        switch (D) {
            case 1: return launch13<T, 1, 2, E>;
            case 2: return launch13<T, 2, 2, E>;
            case 3: return launch13<T, 3, 2, E>;
            case 4: return launch13<T, 4, 2, E>;
            default: return nullptr;
        }
    }
    return nullptr;
}

}  // namespace

// compiled variants: VY = 4 rows per thread (dim_T <= 2), VY = 2 (dim_T <= 4); 256 threads max
St13LaunchFn st13_lookup(int dtype, bool exact, int D, int VY) {
    if (dtype == 0) return exact ? pick13<float, true>(D, VY) : pick13<float, false>(D, VY);
    return exact ? pick13<double, true>(D, VY) : pick13<double, false>(D, VY);
}

}  // namespace st35d
