// SoA multi-stream copy microbenchmark (diagnostics, not product): the data
// movement of one D3Q19 step without the collision — read Q populations of a
// cell (SoA, population stride = the lattice size) and write them back at the
// same cell of a second lattice.  Measures what HBM delivers for the LBM's
// 2 x 19-stream access pattern (the roof the LBM kernels are held against).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 tools/soa_copy.cu -o /tmp/soa_copy
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

template <int Q, int V>
__global__ void __launch_bounds__(256) soa_copy(const float* __restrict__ a, float* __restrict__ b, size_t n, size_t pad) {
    const size_t stride = n + pad;
    const size_t nv = n / V;
    for (size_t t = blockIdx.x * (size_t)blockDim.x + threadIdx.x; t < nv; t += (size_t)gridDim.x * blockDim.x) {
        if (V == 4) {
            float4 v[Q];
#pragma unroll
            for (int i = 0; i < Q; ++i) v[i] = reinterpret_cast<const float4*>(a + i * stride)[t];
#pragma unroll
            for (int i = 0; i < Q; ++i) reinterpret_cast<float4*>(b + i * stride)[t] = v[i];
        } else {
            float v[Q];
#pragma unroll
            for (int i = 0; i < Q; ++i) v[i] = a[i * stride + t];
#pragma unroll
            for (int i = 0; i < Q; ++i) b[i * stride + t] = v[i];
        }
    }
}

template <int Q, int V>
static void run(const char* name, float* a, float* b, size_t n, size_t pad, int bps) {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int grid = sms * bps;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int w = 0; w < 3; ++w) soa_copy<Q, V><<<grid, 256>>>(a, b, n, pad);
    const int R = 10;
    cudaEventRecord(e0);
    for (int r = 0; r < R; ++r) soa_copy<Q, V><<<grid, 256>>>(a, b, n, pad);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    const double bytes = 2.0 * Q * n * 4 * R;
    printf("%-28s Q=%2d V=%d pad=%6zu ctas/SM=%d: %7.1f GB/s\n", name, Q, V, pad, bps, bytes / (ms * 1e-3) / 1e9);
}

int main() {
    const size_t n = 256ull * 256 * 256;
    float *a, *b;
    const size_t maxpad = 4096;
    cudaMalloc(&a, 19 * (n + maxpad) * 4);
    cudaMalloc(&b, 19 * (n + maxpad) * 4);
    cudaMemset(a, 0, 19 * (n + maxpad) * 4);
    for (int bps : {4, 8}) {
        run<1, 4>("1 stream (memcpy)", a, b, 19 * n, 0, bps);
        run<19, 1>("19 streams scalar", a, b, n, 0, bps);
        run<19, 4>("19 streams float4", a, b, n, 0, bps);
        run<19, 1>("19 streams scalar pad", a, b, n, 1024, bps);
        run<19, 4>("19 streams float4 pad", a, b, n, 1024, bps);
        run<19, 1>("19 streams scalar pad", a, b, n, 4096 - 64, bps);
    }
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) printf("error %s\n", cudaGetErrorString(e));
    return 0;
}
