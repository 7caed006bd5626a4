// lbm_inst.cu — instantiates the LBM kernels and the shell-flag check.
#include "launch.h"

namespace st35d {

template <typename T, bool E>
static cudaError_t push_t(const void* src, void* dst, const uint8_t* flags, const LbmParams& p, int grid,
                          cudaStream_t s) {
    lbm_push_kernel<T, E><<<grid, 256, 0, s>>>(static_cast<const T*>(src), static_cast<T*>(dst), flags, p);
    return cudaGetLastError();
}

cudaError_t lbm_push_launch(int dtype, bool exact, const void* src, void* dst, const uint8_t* flags,
                            const LbmParams& p, int grid, cudaStream_t s) {
    if (dtype == 0) return exact ? push_t<float, true>(src, dst, flags, p, grid, s)
                                 : push_t<float, false>(src, dst, flags, p, grid, s);
    return exact ? push_t<double, true>(src, dst, flags, p, grid, s)
                 : push_t<double, false>(src, dst, flags, p, grid, s);
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
