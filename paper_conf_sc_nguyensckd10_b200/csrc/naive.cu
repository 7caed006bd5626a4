// naive.cu — the "no blocking" 7-point baseline of the ablation ladder
// (Fig. 5(b): "no blocking" is the first
// bar).  One Jacobi step per launch, one thread per point, all
// seven inputs read from global memory: the only reuse is what L1/L2 give,
// i.e. what the 2.5D / 3.5D sweeps are measured against.  The arithmetic is
// the oracle's order with every operation rounded (X2), so the result is
// bit-identical to the oracle in both builds.  Not a product path: selected
// only by st_plan_set_variant(plan, ST_VARIANT_NAIVE).
#include "launch.h"

namespace st35d {

template <typename T> struct Rn;
template <> struct Rn<float> {
    static __device__ __forceinline__ float add(float a, float b) { return __fadd_rn(a, b); }
    static __device__ __forceinline__ float mul(float a, float b) { return __fmul_rn(a, b); }
};
template <> struct Rn<double> {
    static __device__ __forceinline__ double add(double a, double b) { return __dadd_rn(a, b); }
    static __device__ __forceinline__ double mul(double a, double b) { return __dmul_rn(a, b); }
};

// grid (ceil(nx / 128), ny, nz): no index divisions
template <typename T>
__global__ void __launch_bounds__(128) st7_naive_kernel(const T* __restrict__ a, T* __restrict__ b, int nx, int ny,
                                                         int nz, double alpha, double beta) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y, z = blockIdx.z;
    if (x >= nx) return;
    const size_t plane = (size_t)nx * ny;
    const size_t c = (size_t)z * plane + (size_t)y * nx + x;
    const T v = a[c];
    if (x == 0 || y == 0 || z == 0 || x == nx - 1 || y == ny - 1 || z == nz - 1) {   // Dirichlet shell (X1)
        b[c] = v;
        return;
    }
    using R = Rn<T>;
    const T sx = R::add(a[c - 1], a[c + 1]);
    const T sy = R::add(a[c - nx], a[c + nx]);
    const T sz = R::add(a[c - plane], a[c + plane]);
    const T s = R::add(R::add(sx, sy), sz);
    b[c] = R::add(R::mul(T(alpha), v), R::mul(T(beta), s));
}

cudaError_t st7_naive_launch(int dtype, const void* in, void* out, int nx, int ny, int nz, double alpha, double beta,
                             cudaStream_t s) {
    if (ny > 65535 || nz > 65535) return cudaErrorInvalidValue;
    const dim3 grid((nx + 127) / 128, ny, nz);
    if (dtype == 0)
        st7_naive_kernel<float><<<grid, 128, 0, s>>>(static_cast<const float*>(in), static_cast<float*>(out), nx, ny,
                                                     nz, (double)(float)alpha, (double)(float)beta);
    else
        st7_naive_kernel<double><<<grid, 128, 0, s>>>(static_cast<const double*>(in), static_cast<double*>(out), nx,
                                                      ny, nz, alpha, beta);
    return cudaGetLastError();
}

}  // namespace st35d
