// microbench.cu — per-SM throughput of the instructions the 7-point / LBM
// sweeps are built from (FP32/FP64 pipes, packed f32x2, SHFL, LDS/STS.128).
// Output: lane-ops (or bytes) per SM clock, measured with clock64 inside a
// single resident wave.  Used to set the ALU roofline in DESIGN.md.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

constexpr int ITERS = 4096;

__device__ unsigned long long g_cycles[4096];
__device__ float g_sinkf[1 << 20];
__device__ double g_sinkd[1 << 20];

__device__ unsigned long long g_ns[4096];
__device__ __forceinline__ unsigned long long gtimer() { unsigned long long t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t; }
// clock64 (SM cycles) and %globaltimer (ns) over the same region: their ratio is the
// SM clock the region actually ran at (round 1 divided by the event time of the whole
// launch instead, which under-estimated the clock and gave impossible >128 lanes/clk)
#define TIMED_BEGIN  __syncthreads(); long long t0 = clock64(); unsigned long long n0 = gtimer();
#define TIMED_END    __syncthreads(); long long t1 = clock64(); unsigned long long n1 = gtimer(); \
    if (threadIdx.x == 0) { g_cycles[blockIdx.x] = t1 - t0; g_ns[blockIdx.x] = n1 - n0; }

__global__ void k_ffma(float a, float b) {
    float x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            x0 = fmaf(x0, a, b); x1 = fmaf(x1, a, b); x2 = fmaf(x2, a, b); x3 = fmaf(x3, a, b);
            x4 = fmaf(x4, a, b); x5 = fmaf(x5, a, b); x6 = fmaf(x6, a, b); x7 = fmaf(x7, a, b);
        }
    }
    TIMED_END
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

__global__ void k_fadd(float a, float b) {
    float x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
    float y = a * b;
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            x0 = x0 + y; x1 = x1 + x0; x2 = x2 + y; x3 = x3 + x2;
            x4 = x4 + y; x5 = x5 + x4; x6 = x6 + y; x7 = x7 + x6;
        }
    }
    TIMED_END
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

__device__ __forceinline__ void fadd2(float& a0, float& a1, float b0, float b1) {
    unsigned long long A, B;
    asm("mov.b64 %0, {%1,%2};" : "=l"(A) : "f"(a0), "f"(a1));
    asm("mov.b64 %0, {%1,%2};" : "=l"(B) : "f"(b0), "f"(b1));
    asm("add.rn.f32x2 %0, %0, %1;" : "+l"(A) : "l"(B));
    asm("mov.b64 {%0,%1}, %2;" : "=f"(a0), "=f"(a1) : "l"(A));
}
__device__ __forceinline__ void ffma2(float& a0, float& a1, float b0, float b1, float c0, float c1) {
    unsigned long long A, B, C;
    asm("mov.b64 %0, {%1,%2};" : "=l"(A) : "f"(a0), "f"(a1));
    asm("mov.b64 %0, {%1,%2};" : "=l"(B) : "f"(b0), "f"(b1));
    asm("mov.b64 %0, {%1,%2};" : "=l"(C) : "f"(c0), "f"(c1));
    asm("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(A) : "l"(B), "l"(C));
    asm("mov.b64 {%0,%1}, %2;" : "=f"(a0), "=f"(a1) : "l"(A));
}

__global__ void k_fadd2(float a, float b) {
    float x[16];
#pragma unroll
    for (int j = 0; j < 16; ++j) x[j] = threadIdx.x + j;
    float y0 = a * b, y1 = a + b;
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 16; j += 2) fadd2(x[j], x[j + 1], y0, y1);
#pragma unroll
        for (int j = 0; j < 16; j += 2) fadd2(x[j], x[j + 1], y1, y0);
    }
    TIMED_END
    float s = 0;
#pragma unroll
    for (int j = 0; j < 16; ++j) s += x[j];
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_ffma2(float a, float b) {
    float x[16];
#pragma unroll
    for (int j = 0; j < 16; ++j) x[j] = threadIdx.x + j;
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 16; j += 2) ffma2(x[j], x[j + 1], a, b, b, a);
#pragma unroll
        for (int j = 0; j < 16; j += 2) ffma2(x[j], x[j + 1], b, a, a, b);
    }
    TIMED_END
    float s = 0;
#pragma unroll
    for (int j = 0; j < 16; ++j) s += x[j];
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_dfma(double a, double b) {
    double x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            x0 = fma(x0, a, b); x1 = fma(x1, a, b); x2 = fma(x2, a, b); x3 = fma(x3, a, b);
            x4 = fma(x4, a, b); x5 = fma(x5, a, b); x6 = fma(x6, a, b); x7 = fma(x7, a, b);
        }
    }
    TIMED_END
    g_sinkd[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

__global__ void k_dadd(double a, double b) {
    double x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
    double y = a * b;
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            x0 = x0 + y; x1 = x1 + x0; x2 = x2 + y; x3 = x3 + x2;
            x4 = x4 + y; x5 = x5 + x4; x6 = x6 + y; x7 = x7 + x6;
        }
    }
    TIMED_END
    g_sinkd[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

__global__ void k_shfl(float a, float b) {
    float x0 = threadIdx.x * a, x1 = x0 + b, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            x0 = __shfl_down_sync(0xffffffffu, x0, 1); x1 = __shfl_up_sync(0xffffffffu, x1, 1);
            x2 = __shfl_down_sync(0xffffffffu, x2, 1); x3 = __shfl_up_sync(0xffffffffu, x3, 1);
            x4 = __shfl_down_sync(0xffffffffu, x4, 1); x5 = __shfl_up_sync(0xffffffffu, x5, 1);
            x6 = __shfl_down_sync(0xffffffffu, x6, 1); x7 = __shfl_up_sync(0xffffffffu, x7, 1);
        }
    }
    TIMED_END
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

// FADD and SHFL interleaved 4:1 — do they co-issue without stealing FP throughput?
__global__ void k_fadd_shfl(float a, float b) {
    float x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
    float s0 = a, s1 = b;
    float y = a * b;
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            x0 = x0 + y; x1 = x1 + x0; x2 = x2 + y; x3 = x3 + x2;
            s0 = __shfl_down_sync(0xffffffffu, s0, 1);
            x4 = x4 + y; x5 = x5 + x4; x6 = x6 + y; x7 = x7 + x6;
            s1 = __shfl_up_sync(0xffffffffu, s1, 1);
        }
    }
    TIMED_END
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7 + s0 + s1;
}

__global__ void k_lds128(float a, float b) {
    extern __shared__ float4 sm[];
    int n = blockDim.x;
    sm[threadIdx.x] = make_float4(a, b, a, b);
    float4 acc = make_float4(0, 0, 0, 0);
    int idx = threadIdx.x;
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            float4 v = sm[(idx + j * 32 + i * 64) & (n - 1)];
            acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;  // 4 fadd per LDS.128
        }
    }
    TIMED_END
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = acc.x + acc.y + acc.z + acc.w;
}

__global__ void k_sts128(float a, float b) {
    extern __shared__ float4 sm[];
    int n = blockDim.x;
    float4 v = make_float4(a, b, a + threadIdx.x, b);
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) { sm[(threadIdx.x + j * 32) & (n - 1)] = v; v.x += 1.0f; }
    }
    TIMED_END
    __syncthreads();
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = sm[threadIdx.x].x;
}


// Packed FP32 with DISTINCT register operands every instruction (no operand
// reuse), the stencil's pattern: does the register file sustain 2 pair reads
// (FADD2) / 3 pair reads (FFMA2) per instruction at full rate?
__global__ void k_fadd2_distinct(float a, float b) {
    float2 x[24];
#pragma unroll
    for (int j = 0; j < 24; ++j) x[j] = make_float2(threadIdx.x + j, a + j);
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = __fadd2_rn(x[j + 8], x[j + 16]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j + 8] = __fadd2_rn(x[j + 16], x[j]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j + 16] = __fadd2_rn(x[j], x[j + 8]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = __fadd2_rn(x[j + 8], x[j + 16]);
    }
    TIMED_END
    float s = 0;
#pragma unroll
    for (int j = 0; j < 24; ++j) s += x[j].x + x[j].y;
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_ffma2_distinct(float a, float b) {
    float2 x[24];
#pragma unroll
    for (int j = 0; j < 24; ++j) x[j] = make_float2(threadIdx.x + j, a + j);
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = __ffma2_rn(x[j + 8], x[j + 16], x[j]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j + 8] = __ffma2_rn(x[j + 16], x[j], x[j + 8]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j + 16] = __ffma2_rn(x[j], x[j + 8], x[j + 16]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = __ffma2_rn(x[j + 8], x[j + 16], x[j]);
    }
    TIMED_END
    float s = 0;
#pragma unroll
    for (int j = 0; j < 24; ++j) s += x[j].x + x[j].y;
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_fadd_distinct(float a, float b) {
    float x[24];
#pragma unroll
    for (int j = 0; j < 24; ++j) x[j] = threadIdx.x + j * a;
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = __fadd_rn(x[j + 8], x[j + 16]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j + 8] = __fadd_rn(x[j + 16], x[j]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j + 16] = __fadd_rn(x[j], x[j + 8]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = __fadd_rn(x[j + 8], x[j + 16]);
    }
    TIMED_END
    float s = 0;
#pragma unroll
    for (int j = 0; j < 24; ++j) s += x[j];
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = s;
}


// FFMA2 / FMUL2 with one SCALAR (broadcast) operand and distinct pairs
__global__ void k_ffma2_scalar(float a, float b) {
    float2 x[24];
#pragma unroll
    for (int j = 0; j < 24; ++j) x[j] = make_float2(threadIdx.x + j, a + j);
    const float2 c = make_float2(a, a);
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = __ffma2_rn(c, x[j + 8], x[j + 16]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j + 8] = __ffma2_rn(c, x[j + 16], x[j]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j + 16] = __ffma2_rn(c, x[j], x[j + 8]);
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = __ffma2_rn(c, x[j + 8], x[j + 16]);
    }
    TIMED_END
    float s = 0;
#pragma unroll
    for (int j = 0; j < 24; ++j) s += x[j].x + x[j].y;
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// the 7-point update mix per point pair: 4 FADD2 (distinct pairs), FMUL2 and
// 2 FFMA2 with a scalar coefficient
__global__ void k_mix7(float a, float b) {
    float2 x[24];
#pragma unroll
    for (int j = 0; j < 24; ++j) x[j] = make_float2(threadIdx.x + j, a + j);
    const float2 al = make_float2(a, a), be = make_float2(b, b);
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const float2 s1 = __fadd2_rn(x[j], x[j + 8]);
            const float2 s2 = __fadd2_rn(x[j + 16], x[(j + 1) % 8]);
            const float2 s3 = __fadd2_rn(s1, x[(j + 3) % 8 + 8]);
            const float2 s = __fadd2_rn(s3, s2);
            const float2 t = __ffma2_rn(al, x[j + 16], __fmul2_rn(be, s));
            x[j + 16] = __ffma2_rn(be, x[(j + 5) % 8 + 8], t);
        }
    }
    TIMED_END
    float s = 0;
#pragma unroll
    for (int j = 0; j < 24; ++j) s += x[j].x + x[j].y;
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// the same mix with per-element coefficient PAIRS (3 register pairs per FFMA2)
__global__ void k_mix7_pairs(float a, float b) {
    float2 x[24];
#pragma unroll
    for (int j = 0; j < 24; ++j) x[j] = make_float2(threadIdx.x + j, a + j);
    const float2 al = make_float2(a, a + threadIdx.x * 1e-9f), be = make_float2(b, b - threadIdx.x * 1e-9f);
    TIMED_BEGIN
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const float2 s1 = __fadd2_rn(x[j], x[j + 8]);
            const float2 s2 = __fadd2_rn(x[j + 16], x[(j + 1) % 8]);
            const float2 s3 = __fadd2_rn(s1, x[(j + 3) % 8 + 8]);
            const float2 s = __fadd2_rn(s3, s2);
            const float2 t = __ffma2_rn(al, x[j + 16], __fmul2_rn(be, s));
            x[j + 16] = __ffma2_rn(be, x[(j + 5) % 8 + 8], t);
        }
    }
    TIMED_END
    float s = 0;
#pragma unroll
    for (int j = 0; j < 24; ++j) s += x[j].x + x[j].y;
    g_sinkf[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <typename K>
static int run(const char* name, K kern, int threads, double ops_per_thread_iter, int blocks_per_sm, size_t smem = 0) {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    int blocks = nsm * blocks_per_sm;
    if (smem) cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    kern<<<blocks, threads, smem>>>(1.0000001f, 0.999999f);  // warm-up
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<<<blocks, threads, smem>>>(1.0000001f, 0.999999f);
    cudaEventRecord(e1);
    CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    unsigned long long cyc[4096];
    CK(cudaMemcpyFromSymbol(cyc, g_cycles, sizeof(unsigned long long) * blocks));
    unsigned long long ns[4096];
    CK(cudaMemcpyFromSymbol(ns, g_ns, sizeof(unsigned long long) * blocks));
    double mean = 0, mns = 0; for (int i = 0; i < blocks; ++i) { mean += cyc[i]; mns += ns[i]; } mean /= blocks; mns /= blocks;
    double ops_per_sm = ops_per_thread_iter * ITERS * threads * blocks_per_sm;
    // whole-launch throughput: every CTA's work over the event time (CTAs are not
    // evenly co-resident, so per-CTA clock windows overstate the per-SM rate)
    const double ev = ops_per_sm * nsm / (ms * 1e-3) / nsm / (mean / mns * 1e9);
    printf("%-16s threads=%4d bps=%d  %8.2f lane-ops/clk/SM (whole launch, events)  clk %.0f MHz  %.3f ms\n",
           name, threads, blocks_per_sm, ev, mean / mns * 1e3, ms);
    return 0;
}

template <typename K>
static int rund(const char* name, K kern, int threads, double ops, int bps) {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    int blocks = nsm * bps;
    kern<<<blocks, threads>>>(1.0000001, 0.999999);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<<<blocks, threads>>>(1.0000001, 0.999999);
    cudaEventRecord(e1);
    CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    unsigned long long cyc[4096];
    CK(cudaMemcpyFromSymbol(cyc, g_cycles, sizeof(unsigned long long) * blocks));
    unsigned long long ns[4096];
    CK(cudaMemcpyFromSymbol(ns, g_ns, sizeof(unsigned long long) * blocks));
    double mean = 0, mns = 0; for (int i = 0; i < blocks; ++i) { mean += cyc[i]; mns += ns[i]; } mean /= blocks; mns /= blocks;
    printf("%-14s threads=%4d bps=%d  %8.2f lane-ops/clk/SM  %8.2f lane-ops/ns/SM  (clk %.0f MHz from clock64/globaltimer, %.3f ms)\n",
           name, threads, bps, ops * ITERS * threads * bps / mean, ops * ITERS * threads * bps / mns, mean / mns * 1e3, ms);
    return 0;
}

int main() {
    cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
    printf("device %s, %d SMs, smem/block optin %zu, regs/SM %d, L2 %d\n", p.name, p.multiProcessorCount,
           p.sharedMemPerBlockOptin, p.regsPerMultiprocessor, p.l2CacheSize);
    for (int t : {256, 512}) {
        run("ffma", k_ffma, t, 32, 2);
        run("fadd", k_fadd, t, 32, 2);
        run("fadd2(x2)", k_fadd2, t, 32, 2);
        run("ffma2(x2)", k_ffma2, t, 32, 2);
        run("fadd2 distinct", k_fadd2_distinct, t, 64, 2);
        run("ffma2 distinct", k_ffma2_distinct, t, 64, 2);
        run("fadd distinct", k_fadd_distinct, t, 32, 2);
        run("ffma2 scalar", k_ffma2_scalar, t, 64, 2);
        run("mix7 scalar", k_mix7, t, 8 * 14, 2);
        run("mix7 pairs", k_mix7_pairs, t, 8 * 14, 2);
        rund("dfma", k_dfma, t, 32, 2);
        rund("dadd", k_dadd, t, 32, 2);
        run("shfl", k_shfl, t, 32, 2);
        run("fadd+shfl", k_fadd_shfl, t, 40, 2);   // 32 fadd + 8 shfl per iter
        run("lds128(+4fadd)", k_lds128, t, 8, 2, t * 16);  // LDS.128 per clk (x4 = words)
        run("sts128", k_sts128, t, 8, 2, t * 16);
    }
    return 0;
}
