// st7_inst.cu — instantiates st7_35d_kernel for one (dtype, mode); compiled
// once per combination with -DST_T=float|double -DST_EXACT=0|1.
#include "launch.h"
#include "st7_split.cuh"

#ifndef ST_T
#define ST_T float
#endif
#ifndef ST_EXACT
#define ST_EXACT 0
#endif

#define ST_CAT2(a, b) a##b
#define ST_CAT(a, b) ST_CAT2(a, b)
#if ST_EXACT
#define ST_MODE exact
#else
#define ST_MODE fast
#endif
// a NAMED per-unit namespace: nvcc emits template instantiations inside an
// anonymous namespace as weak symbols with identical names in every unit,
// which the linker would merge across the four (dtype, mode) objects.
#define ST_UNIT_NS ST_CAT(ST_CAT(ST_CAT(unit_, ST_TNAME), _), ST_MODE)

namespace st35d {
namespace ST_UNIT_NS {

using TT = ST_T;
constexpr int NTX = sizeof(TT) == 4 ? 16 : 32;

template <int D, int VY, int MAXT>
cudaError_t launch(const CUtensorMap* map, const St7Params& p, int grid, int threads, size_t smem,
                   cudaStream_t s) {
    auto k = st7_35d_kernel<TT, D, NTX, VY, ST_EXACT != 0, MAXT>;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return launch_pdl(k, grid, threads, smem, s, *map, p);
}

template <int VY, int MAXT>
St7LaunchFn pick(int D) {
    switch (D) {
        case 1: return launch<1, VY, MAXT>;
        case 2: return launch<2, VY, MAXT>;
        case 3: return launch<3, VY, MAXT>;
        case 4: return launch<4, VY, MAXT>;
        case 5: return launch<5, VY, MAXT>;
        case 6: return launch<6, VY, MAXT>;
        case 7: return launch<7, VY, MAXT>;
        case 8: return launch<8, VY, MAXT>;
        default: return nullptr;
    }
}

template <int D, int VY, int MAXT>
cudaError_t launch_split(const CUtensorMap* map, const St7Params& p, int grid, int threads, size_t smem,
                         cudaStream_t s) {
    auto k = st7_35d_split_kernel<TT, D, (D + 1) / 2, NTX, VY, ST_EXACT != 0, MAXT>;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k<<<grid, threads, smem, s>>>(*map, p);
    return cudaGetLastError();
}

template <int VY, int MAXT>
St7LaunchFn pick_split(int D) {
    switch (D) {
        case 2: return launch_split<2, VY, MAXT>;
        case 3: return launch_split<3, VY, MAXT>;
        case 4: return launch_split<4, VY, MAXT>;
        case 5: return launch_split<5, VY, MAXT>;
        case 6: return launch_split<6, VY, MAXT>;
        default: return nullptr;
    }
}

}  // namespace ST_UNIT_NS
using namespace ST_UNIT_NS;

#define ST_FN ST_CAT(ST_CAT(ST_CAT(st7_lookup_, ST_TNAME), _), ST_MODE)

// variants: (VY=4, 256 threads max), (VY=2, 256), (VY=2, 512 threads: <= 128 registers)
St7LaunchFn ST_FN(int D, int VY, int MAXT) {
    if (VY == 4 && MAXT == 256) return pick<4, 256>(D);
    if (VY == 2 && MAXT == 256) return pick<2, 256>(D);
    if (VY == 2 && MAXT == 512) return pick<2, 512>(D);
    if (VY == 4 && MAXT == 384) return pick<4, 384>(D);
    return nullptr;
}

}  // namespace st35d

namespace st35d {
#define ST_SFN ST_CAT(ST_CAT(ST_CAT(st7s_lookup_, ST_TNAME), _), ST_MODE)
St7LaunchFn ST_SFN(int D, int VY, int MAXT) {
    if (VY == 2 && MAXT == 512) return pick_split<2, 512>(D);
    if (VY == 4 && MAXT == 384) return pick_split<4, 384>(D);
    return nullptr;
}
}  // namespace st35d
