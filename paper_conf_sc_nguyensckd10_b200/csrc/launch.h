// launch.h — internal dispatch between the C-ABI (api.cu) and the kernel
// instantiation units (st7_inst.cu compiled per dtype/mode, lbm_inst.cu).
#pragma once
#include <cstdlib>
#include <cuda.h>
#include <cuda_runtime.h>
#include "st7_kernel.cuh"
#include "lbm_kernel.cuh"

namespace st35d {

// launch with programmatic stream serialization (PDL): the kernel's prologue may
// overlap the previous kernel in the stream; the kernel orders its memory
// accesses after it with griddepcontrol.wait (pdl = false: plain launch, ST_OPT_PDL A/B)
template <typename K, typename... A>
inline cudaError_t launch_pdl(bool pdl, K kernel, int grid, int threads, size_t smem, cudaStream_t s, A... args) {
    const bool off = !pdl;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = off ? 0 : 1;
    return cudaLaunchKernelEx(&cfg, kernel, args...);
}

using St7LaunchFn = cudaError_t (*)(const CUtensorMap* map, const St7Params& p, int grid, int threads,
                                    size_t smem, cudaStream_t s);

// returns nullptr if (D, VY, NT, MINB, VX) is not compiled (VX 0: the dtype's 16-byte vector)
St7LaunchFn st7_lookup_f32_fast(int D, int VY, int NT, int MINB, int VX);
St7LaunchFn st7_lookup_f32_exact(int D, int VY, int NT, int MINB, int VX);
St7LaunchFn st7_lookup_f64_fast(int D, int VY, int NT, int MINB, int VX);
St7LaunchFn st7_lookup_f64_exact(int D, int VY, int NT, int MINB, int VX);

// radius-2 (13-point star) sweep (st13_kernel.cuh); nullptr if (D, VY) is not compiled
struct St13Params;
using St13LaunchFn = cudaError_t (*)(const CUtensorMap* map, const St13Params& p, int grid, int threads, size_t smem,
                                     cudaStream_t s);
St13LaunchFn st13_lookup(int dtype, bool exact, int D, int VY);
constexpr int ST13_MAX_DIM_T = 4;

// 27-point sweep on the 7-point machinery (st27t_kernel.cuh, tolerance build);
// nullptr if (D, VY) is not compiled
struct St27tParams;
using St27tLaunchFn = cudaError_t (*)(const CUtensorMap* map, const St27tParams& p, int grid, int threads,
                                      size_t smem, cudaStream_t s);
St27tLaunchFn st27t_lookup(int dtype, int D, int VY);
constexpr int ST27T_MAX_DIM_T = 4;
// VY = 4 rows per thread up to this depth, else 2 (measured 256^3 FP32 dim_T 2: VY 2 623,
// VY 4 524 Gupd/s -- 255 registers with spills)
constexpr int ST27T_VY4_MAX = 1;

bool lbm_push_batched(int esize, int nx, int ny, int nzb, int force);   // kernel choice (also sets the grid)
cudaError_t lbm_push_launch(int dtype, bool exact, bool slab, bool batched, const void* src, void* dst,
                            const uint8_t* fl2, const LbmParams& p, int grid, cudaStream_t s);
cudaError_t lbm_gather_launch(int dtype, bool exact, int mode, const void* src, void* dst, const uint8_t* fl2,
                              const LbmParams& p, int grid, cudaStream_t s);
// TMA-fed pull pass of the gather form (lbm_tma.cu); maps = two 3D (x, y, 19 nz)
// tensor maps of the source lattice, boxes (bx, by, 1) and (bx + halo, by, 1)
size_t lbm_pull_tma_stage_bytes(int dtype, int nx);
void lbm_pull_tma_box(int dtype, int nx, int* bx, int* by, int* halo);
// mode: LBM_COLLIDE / LBM_PULL / LBM_STREAM (the gather form's three passes)
cudaError_t lbm_pull_tma_launch(int dtype, bool exact, int mode, bool pdl, const CUtensorMap* maps, const void* src,
                                void* dst, const uint8_t* fl2, const LbmParams& p, int grid, int stages,
                                cudaStream_t s);
cudaError_t lbm35_launch(int dtype, bool exact, int D, const Lbm35Params& p, int grid, int threads, size_t smem,
                         cudaStream_t s);
cudaError_t st7_naive_launch(int dtype, const void* in, void* out, int nx, int ny, int nz, double alpha,
                             double beta, cudaStream_t s);
cudaError_t lbm_fl2(const uint8_t* flags, uint8_t* fl2, int nx, int ny, int nz, cudaStream_t s);
constexpr int LBM35_MAX_D = 3;
cudaError_t lbm_shell_check(const uint8_t* flags, int nx, int ny, int nz, int* d_count, cudaStream_t s);

// 27-point 3.5D sweep (st27.cu), depth D in [1, st27_depth_max()]; grid_out = CTAs launched
int st27_depth_max(int dtype);
cudaError_t st27_launch(int dtype, bool exact, int D, const void* in, void* out, int nx, int ny, int nz, double alpha,
                        double beta, double gamma, double delta, int sms, cudaStream_t s, int* grid_out);

}  // namespace st35d
