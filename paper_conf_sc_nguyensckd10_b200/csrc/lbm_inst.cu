// lbm_inst.cu — instantiates the LBM kernels and the shell-flag check.
#include <cstdlib>
#include "launch.h"

namespace st35d {

// FP32 lattices of more than 2^24 cells run the batched-flag kernel (3 CTAs/SM):
// it holds 25-28 GLUPS from 320^3 to 1024^3 (25.4 vs 15.4 at 1024^3, 25.6 vs
// 18.5 at 512^3), while the per-direction kernel at 4 CTAs/SM swings with the
// lattice size and only matches it up to 256^3 (tools/lbm_big.py, T = 20);
// FP64 always batches (2 CTAs/SM).  force = 0/1 overrides (st_plan_set_option
// ST_OPT_LBM_BATCHED, used by the parity tests to reach both kernels).
bool lbm_push_batched(int esize, int nx, int ny, int nzb, int force) {
    if (force >= 0) return force != 0 || esize == 8;
    return esize == 8 || (long long)nx * ny * nzb > (1LL << 24);
}

template <typename T, bool E, bool SLAB>
static cudaError_t push_t(bool batched, const void* src, void* dst, const uint8_t* fl2, const LbmParams& p, int grid,
                          cudaStream_t s) {
    // FP64: 32-bit element offsets when every population offset (and a plane step)
    // fits; FP32 keeps 64-bit offsets (measured 26.0 vs 23.6 GLUPS at 256^3, tools/lbm_ab.sh)
    const long long span = 20LL * p.nx * p.ny * p.nzb;
    const T* a = static_cast<const T*>(src);
    T* b = static_cast<T*>(dst);
    if (sizeof(T) == 8) {
        if (span < (1LL << 31)) lbm_push_kernel<T, E, int, true, SLAB><<<grid, 256, 0, s>>>(a, b, fl2, p);
        else lbm_push_kernel<T, E, long long, true, SLAB><<<grid, 256, 0, s>>>(a, b, fl2, p);
    } else if (batched) {
        lbm_push_kernel<T, E, long long, true, SLAB><<<grid, 256, 0, s>>>(a, b, fl2, p);
    } else {
        lbm_push_kernel<T, E, long long, false, SLAB><<<grid, 256, 0, s>>>(a, b, fl2, p);
    }
    return cudaGetLastError();
}

template <typename T, bool E>
static cudaError_t push_s(bool slab, bool batched, const void* src, void* dst, const uint8_t* fl2, const LbmParams& p,
                          int grid, cudaStream_t s) {
    return slab ? push_t<T, E, true>(batched, src, dst, fl2, p, grid, s)
                : push_t<T, E, false>(batched, src, dst, fl2, p, grid, s);
}

// fl2 = the lbm_fl2 prepass output of the flags; batched = lbm_push_batched(...)
cudaError_t lbm_push_launch(int dtype, bool exact, bool slab, bool batched, const void* src, void* dst,
                            const uint8_t* fl2, const LbmParams& p, int grid, cudaStream_t s) {
    if (dtype == 0) return exact ? push_s<float, true>(slab, batched, src, dst, fl2, p, grid, s)
                                 : push_s<float, false>(slab, batched, src, dst, fl2, p, grid, s);
    return exact ? push_s<double, true>(slab, batched, src, dst, fl2, p, grid, s)
                 : push_s<double, false>(slab, batched, src, dst, fl2, p, grid, s);
}

template <typename T, bool E>
static cudaError_t gather_t(int mode, const void* src, void* dst, const uint8_t* fl2, const LbmParams& p, int grid,
                            cudaStream_t s) {
    const T* a = static_cast<const T*>(src);
    T* b = static_cast<T*>(dst);
    if (mode == LBM_COLLIDE) lbm_gather_kernel<T, E, LBM_COLLIDE><<<grid, 256, 0, s>>>(a, b, fl2, p);
    else if (mode == LBM_PULL) lbm_gather_kernel<T, E, LBM_PULL><<<grid, 256, 0, s>>>(a, b, fl2, p);
    else lbm_gather_kernel<T, E, LBM_STREAM><<<grid, 256, 0, s>>>(a, b, fl2, p);
    return cudaGetLastError();
}

// gather-form passes (mode LBM_COLLIDE / LBM_PULL / LBM_STREAM), single domain
cudaError_t lbm_gather_launch(int dtype, bool exact, int mode, const void* src, void* dst, const uint8_t* fl2,
                              const LbmParams& p, int grid, cudaStream_t s) {
    if (dtype == 0) return exact ? gather_t<float, true>(mode, src, dst, fl2, p, grid, s)
                                 : gather_t<float, false>(mode, src, dst, fl2, p, grid, s);
    return exact ? gather_t<double, true>(mode, src, dst, fl2, p, grid, s)
                 : gather_t<double, false>(mode, src, dst, fl2, p, grid, s);
}

template <typename T, int D, bool E>
static cudaError_t l35_t(const Lbm35Params& p, int grid, int threads, size_t smem, cudaStream_t s) {
    auto k = lbm_35d_kernel<T, D, E>;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k<<<grid, threads, smem, s>>>(p);
    return cudaGetLastError();
}

template <typename T, bool E>
static cudaError_t l35_d(int D, const Lbm35Params& p, int grid, int threads, size_t smem, cudaStream_t s) {
    switch (D) {
        case 1: return l35_t<T, 1, E>(p, grid, threads, smem, s);
        case 2: return l35_t<T, 2, E>(p, grid, threads, smem, s);
        case 3: return l35_t<T, 3, E>(p, grid, threads, smem, s);
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t lbm35_launch(int dtype, bool exact, int D, const Lbm35Params& p, int grid, int threads, size_t smem,
                         cudaStream_t s) {
    if (dtype == 0) return exact ? l35_d<float, true>(D, p, grid, threads, smem, s)
                                 : l35_d<float, false>(D, p, grid, threads, smem, s);
    return exact ? l35_d<double, true>(D, p, grid, threads, smem, s) : l35_d<double, false>(D, p, grid, threads, smem, s);
}

// fl2 = flags | 0x80 where a FLUID cell has a non-FLUID (or out-of-lattice) neighbour
__global__ void lbm_fl2_kernel(const uint8_t* __restrict__ flags, uint8_t* __restrict__ fl2, int nx, int ny, int nz) {
    // grid (ceil(nx / 256), ny, nz): no index divisions
    const int x = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y, z = blockIdx.z;
    if (x >= nx) return;
    const size_t plane = (size_t)nx * ny;
    const size_t c = (size_t)z * plane + (size_t)y * nx + x;
    uint8_t f = flags[c];
    if (f == 0) {
        bool nb = x == 0 || y == 0 || z == 0 || x == nx - 1 || y == ny - 1 || z == nz - 1;
#pragma unroll
        for (int i = 1; i < 19; ++i) {
            if (nb) break;
            nb = flags[(size_t)((long long)c + c_ex[i] + (long long)c_ey[i] * nx + (long long)c_ez[i] * (long long)plane)] != 0;
        }
        if (nb) f |= 0x80;
    }
    fl2[c] = f;
}

cudaError_t lbm_fl2(const uint8_t* flags, uint8_t* fl2, int nx, int ny, int nz, cudaStream_t s) {
    if (nz > 65535 || ny > 65535) return cudaErrorInvalidValue;
    lbm_fl2_kernel<<<dim3((nx + 255) / 256, ny, nz), 256, 0, s>>>(flags, fl2, nx, ny, nz);
    return cudaGetLastError();
}

// counts FLUID cells on the 6 faces of the lattice (the GPU path needs 0)
__global__ void shell_check_kernel(const uint8_t* __restrict__ flags, int nx, int ny, int nz, int* count) {
    const long long nxy = (long long)nx * ny;
    const long long faces = 2 * nxy + 2 * (long long)nx * nz + 2 * (long long)ny * nz;
    int bad = 0;
    for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < faces;
         t += (long long)gridDim.x * blockDim.x) {
        long long x, y, z, u = t;
        if (u < 2 * nxy) { z = u < nxy ? 0 : nz - 1; u %= nxy; y = u / nx; x = u % nx; }
        else if ((u -= 2 * nxy) < 2LL * nx * nz) { long long h = (long long)nx * nz; y = u < h ? 0 : ny - 1; u %= h; z = u / nx; x = u % nx; }
        else { u -= 2LL * nx * nz; long long h = (long long)ny * nz; x = u < h ? 0 : nx - 1; u %= h; z = u / ny; y = u % ny; }
        if (flags[(z * ny + y) * nx + x] == 0) ++bad;
    }
    if (bad) atomicAdd(count, bad);
}

cudaError_t lbm_shell_check(const uint8_t* flags, int nx, int ny, int nz, int* d_count, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(d_count, 0, sizeof(int), s);
    if (e != cudaSuccess) return e;
    shell_check_kernel<<<148, 256, 0, s>>>(flags, nx, ny, nz, d_count);
    return cudaGetLastError();
}

}  // namespace st35d
