// TMA plane-delivery microbenchmark (diagnostics, not product): each CTA streams
// P planes of a bx x by box through a ring of RING slots with PF = RING-2 loads
// in flight, no compute; reports per-plane delivery time vs grid size.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++20 -I paper_conf_sc_nguyensckd10_b200/csrc tools/tma_rate.cu -o tools/tma_rate -lcuda
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <cudaTypedefs.h>
#include "common.cuh"
using namespace st35d;

__global__ void tma_stream(const __grid_constant__ CUtensorMap tmap, int P, int ring, int by, int bx, int n,
                           int tiles, unsigned long long* out, float* sink) {
    extern __shared__ __align__(128) unsigned char smem[];
    float* buf = reinterpret_cast<float*>(smem);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + (size_t)ring * bx * by * 4);
    const int PF = ring - 2;
    const uint32_t bytes = bx * by * 4;
    if (threadIdx.x == 0) { for (int s = 0; s < ring; ++s) mbar_init(&bars[s], 1); fence_mbar_init(); }
    __syncthreads();
    const int t = blockIdx.x % (tiles * tiles);
    const int Lx = (t % tiles) * (bx - 8) - 4, Ly = (t / tiles) * (by - 8) - 4;
    const int z0 = (blockIdx.x / (tiles * tiles)) * 37 % max(1, n - P);
    unsigned long long t0 = 0;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t0));
    if (threadIdx.x == 0)
        for (int q = 0; q < PF && q < P; ++q) {
            mbar_arrive_expect_tx(&bars[q], bytes);
            tma_load_3d(buf + (size_t)q * bx * by, &tmap, &bars[q], Lx, Ly, z0 + q);
        }
    float acc = 0.f;
    unsigned long long tf = 0;
    for (int i = 0; i < P; ++i) {
        const int s = i % ring;
        mbar_wait(&bars[s], (i / ring) & 1);
        if (i == 0) asm volatile("mov.u64 %0, %globaltimer;" : "=l"(tf));
        acc += buf[(size_t)s * bx * by + threadIdx.x];
        __syncthreads();
        if (threadIdx.x == 0 && i + PF < P) {
            const int s2 = (i + PF) % ring;
            mbar_arrive_expect_tx(&bars[s2], bytes);
            tma_load_3d(buf + (size_t)s2 * bx * by, &tmap, &bars[s2], Lx, Ly, z0 + i + PF);
        }
    }
    unsigned long long t1;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t1));
    if (threadIdx.x == 0) { out[blockIdx.x * 3] = t0; out[blockIdx.x * 3 + 1] = tf; out[blockIdx.x * 3 + 2] = t1; }
    if (acc == 12345.f) sink[0] = acc;
}

int main(int argc, char** argv) {
    const int n = 256;
    int bx = argc > 1 ? atoi(argv[1]) : 64, by = argc > 2 ? atoi(argv[2]) : 60;
    int P = argc > 3 ? atoi(argv[3]) : 48, ring = argc > 4 ? atoi(argv[4]) : 11;
    int promo = argc > 5 ? atoi(argv[5]) : 0;
    float* x; cudaMalloc(&x, (size_t)n * n * n * 4); cudaMemset(x, 0, (size_t)n * n * n * 4);
    float* y; cudaMalloc(&y, (size_t)512 << 20);   // L2 flush buffer
    float* sink; cudaMalloc(&sink, 64);
    unsigned long long* out; cudaMalloc(&out, 4096 * 24);
    void* fp = nullptr; cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &q);
    auto enc = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fp);
    CUtensorMap map;
    cuuint64_t dims[3] = {(cuuint64_t)n, (cuuint64_t)n, (cuuint64_t)n};
    cuuint64_t str[2] = {(cuuint64_t)n * 4, (cuuint64_t)n * n * 4};
    cuuint32_t box[3] = {(cuuint32_t)bx, (cuuint32_t)by, 1}, es[3] = {1, 1, 1};
    CUtensorMapL2promotion pr[4] = {CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_64B,
                                    CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B};
    if (enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, x, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_NONE, pr[promo], CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
        printf("encode failed\n"); return 1;
    }
    size_t sm = (size_t)ring * bx * by * 4 + ring * 8;
    cudaFuncSetAttribute(tma_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    const int tiles = (n + bx - 9) / (bx - 8);
    printf("box %dx%d P %d ring %d promo %d smem %zu\n", bx, by, P, ring, promo, sm);
    for (int G : {1, 16, 74, 148}) {
        for (int cold = 0; cold < 2; ++cold) {
            if (cold) cudaMemset(y, cold, (size_t)512 << 20);
            else tma_stream<<<G, 128, sm>>>(map, P, ring, by, bx, n, tiles, out, sink);   // warm L2
            cudaDeviceSynchronize();
            tma_stream<<<G, 128, sm>>>(map, P, ring, by, bx, n, tiles, out, sink);
            cudaError_t e = cudaDeviceSynchronize();
            if (e) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
            std::vector<unsigned long long> h(G * 3);
            cudaMemcpy(h.data(), out, G * 24, cudaMemcpyDeviceToHost);
            unsigned long long mn = ~0ull, mx = 0; double first = 0, per = 0;
            for (int b = 0; b < G; ++b) {
                mn = std::min(mn, h[b * 3]); mx = std::max(mx, h[b * 3 + 2]);
                first += (h[b * 3 + 1] - h[b * 3]) / 1e3 / G;
                per += (h[b * 3 + 2] - h[b * 3 + 1]) / 1e3 / (P - 1) / G;
            }
            double span = (mx - mn) / 1e3;
            printf("G %3d %s: first plane %.2f us, then %.3f us/plane/CTA; aggregate %.0f GB/s\n", G,
                   cold ? "cold" : "warm", first, per, (double)G * P * bx * by * 4 / span / 1e3);
        }
    }
    return 0;
}
