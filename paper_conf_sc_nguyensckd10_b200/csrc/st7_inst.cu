// st7_inst.cu — instantiates the 7-point sweep kernel (st7_kernel.cuh) for one
// (dtype, mode); compiled once per combination with -DST_T=float|double
// -DST_EXACT=0|1 (build.py).
#include "launch.h"

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
constexpr int NTX = sizeof(TT) == 4 ? 16 : 32;   // threads across the 64-point tile row

template <int D, int VY, int NT, int MINB, bool SPLIT = true, int VX = 0>
cudaError_t launch(const CUtensorMap* map, const St7Params& p, int grid, int threads, size_t smem, cudaStream_t s) {
    constexpr int NTXK = VX ? 64 / VX : NTX;
    auto k = st7_35d_kernel<TT, D, NTXK, VY, ST_EXACT != 0, NT, MINB, SPLIT, VX>;
    if (threads > NT || threads % NTXK) return cudaErrorInvalidValue;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return launch_pdl(p.pdl != 0, k, grid, threads, smem, s, *map, p);
}

template <int VY, int NT, int MINB = 1, int VX = 0>
St7LaunchFn pick(int D) {
    switch (D) {
        case 1: return launch<1, VY, NT, MINB, true, VX>;
        case 2: return launch<2, VY, NT, MINB, true, VX>;
        case 3: return launch<3, VY, NT, MINB, true, VX>;
        case 4: return launch<4, VY, NT, MINB, true, VX>;
        case 5: return launch<5, VY, NT, MINB, true, VX>;
        case 6: return launch<6, VY, NT, MINB, true, VX>;
        case 7: return launch<7, VY, NT, MINB, true, VX>;
        case 8: return launch<8, VY, NT, MINB, true, VX>;
        default: return nullptr;
    }
}
template <int VY, int NT, int MINB, bool SPLIT = true, int VX = 0>
St7LaunchFn pick4(int D) {   // shallow sweeps only (register cap 65536 / (NT * MINB))
    switch (D) {
        case 1: return launch<1, VY, NT, MINB, SPLIT, VX>;
        case 2: return launch<2, VY, NT, MINB, SPLIT, VX>;
        case 3: return launch<3, VY, NT, MINB, SPLIT, VX>;
        case 4: return launch<4, VY, NT, MINB, SPLIT, VX>;
        default: return nullptr;
    }
}

}  // namespace ST_UNIT_NS
using namespace ST_UNIT_NS;

#define ST_FN ST_CAT(ST_CAT(ST_CAT(st7_lookup_, ST_TNAME), _), ST_MODE)

// compiled variants (rows per thread VY, threads per CTA NT, CTAs per SM MINB;
// MINB = 9: the level-by-level round order of the ablation ladder): see
// variant_for in api.cu
St7LaunchFn ST_FN(int D, int VY, int NT, int MINB, int VX) {
    if constexpr (sizeof(TT) == 4) {
        if (VX == 2) {   // narrow FP32 layout: 32 threads x 2 points per tile row
            if (MINB == 1 && VY == 4 && NT == 512) return pick<4, 512, 1, 2>(D);
            if (MINB == 1 && VY == 4 && NT == 384) return pick4<4, 384, 1, true, 2>(D);
            if (MINB == 1 && VY == 4 && NT == 256) return pick4<4, 256, 1, true, 2>(D);
            return nullptr;
        }
    }
    if (VX != 0 && VX != (sizeof(TT) == 4 ? 4 : 2)) return nullptr;
#if !ST_EXACT
    if (sizeof(TT) == 4 && MINB == 9 && VY == 4 && NT == 256) return pick4<4, 256, 1, false>(D);   // ladder: no phase split
    if (sizeof(TT) == 4 && MINB == 1 && VY == 1 && NT == 256) return pick4<1, 256, 1>(D);           // ladder: one row per thread
#endif
    if (MINB == 1) {
        if (VY == 4 && NT == 256) return pick<4, 256>(D);
        if (VY == 4 && NT == 384) return pick4<4, 384, 1>(D);
        if (VY == 2 && NT == 256) return pick<2, 256>(D);
        if (VY == 2 && NT == 512) return pick4<2, 512, 1>(D);
    }
    if (MINB == 2 && VY == 2 && NT == 256) return pick4<2, 256, 2>(D);
    return nullptr;
}

#if defined(ST7_TRACE) && !ST_EXACT
extern "C" int ST_CAT(st7_trace_read_, ST_TNAME)(void* host) {   // A/B diagnostics build only
    return (int)cudaMemcpyFromSymbol(host, st7_trace_buf, sizeof(st7_trace_buf));
}
extern "C" int ST_CAT(st7_trace_rounds_, ST_TNAME)(void* host) {
    return (int)cudaMemcpyFromSymbol(host, st7_trace_rnd, sizeof(st7_trace_rnd));
}
extern "C" int ST_CAT(st7_trace_issue_, ST_TNAME)(void* host) {
    return (int)cudaMemcpyFromSymbol(host, st7_trace_iss, sizeof(st7_trace_iss));
}
#endif

}  // namespace st35d
