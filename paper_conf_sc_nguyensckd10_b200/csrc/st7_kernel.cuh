// st7_kernel.cuh — 3.5D-blocked 7-point Jacobi sweep for sm_100a.
//
// Method (§V): an XY sub-plane (tile) is streamed along Z (2.5D
// blocking) while dim_T = D time levels are kept on chip (1D
// temporal blocking); only level 0 is read from HBM and only level
// D is written.  Stencil P:111, fixed boundary P:195 (X1).
//
// B200 mapping (DESIGN.md §6 "7-point kernel"):
//  * persistent CTAs, each taking an equal-cost share of the (tile, z) work
//    items (flexible load balance, P:27 / P:241), split on the host;
//  * level 0: thread 0 issues cp.async.bulk.tensor.3d loads of the TX x TY
//    plane box into a RING-slot shared-memory ring, RING-2 planes ahead, each
//    slot completing on its own mbarrier (the paper's hardware prefetch /
//    explicit global->shared copy);
//  * every thread owns a VX x VY block (VX = one 16-byte vector) at every
//    level and keeps, per level, the planes z-1 and z of its points in
//    registers (the Z neighbours in registers); X neighbours at the block edge
//    come from the adjacent lane by shuffle, Y neighbours at the block edge
//    from the threads above / below through a two-row shared-memory exchange;
//  * lag 1 per level: level l at round r computes plane r-l.  A round runs in
//    two phases.  Phase A forms, for every level independently, the part of
//    the update that does not need this round's new plane:
//        A_l = alpha*H + beta*((y- + y+) + z-) + beta*(x- + x+)
//    (H = centre plane r-l of level l-1, whose in-plane neighbours were
//    exchanged in round r-1).  Phase C adds the z+1 term along the level
//    chain, out_l = A_l + beta*F_l with F_1 = the freshly loaded level-0
//    plane and F_l = out_{l-1}: one FFMA2 per point pair per level, so the
//    levels' in-plane work overlaps and only a D-deep FMA chain is serial.
//    One __syncthreads per round (the exchange rows and the ring slot);
//  * the bit-exact build keeps the oracle order (X2): phase A forms
//    (x- + x+) + (y- + y+) and phase C adds (z- + z+) and the separately
//    rounded products alpha*c + beta*s (scalar __fmul_rn/__fadd_rn: ptxas
//    fuses packed mul+add into FFMA2 even under -fmad=false);
//  * shell points (x, y or z on the grid boundary) are copied (out = H) by
//    warp-uniform fix-ups; halo points beyond the grid read TMA zero fill and
//    never feed a valid point;
//  * the final level is written with 128-bit stores of the written region.
#pragma once
#include <type_traits>
#include "common.cuh"

namespace st35d {

constexpr int ST7_MAX_GRID = 320;   // >= CTAs of one sweep (148 SMs x up to 2 CTAs per SM)
constexpr int ST7_RING_MAX = 12;

struct St7Params {
    void* out;
    int nx, ny;        // plane extent
    int nzb;           // planes in the local buffer (tensor map extent)
    int zbase;         // global z of local plane 0
    int nzg;           // global nz
    int za, zb;        // local output planes [za, zb)
    int tiles_x, ntiles;
    int wx, wy;        // written region per tile (regular tiles)
    int hx;            // x halo (>= D, multiple of VX)
    // y placement (st7_tile): regular tiles iy < tiles_y-1 load rows from
    // iy*wy - D - ey and write [iy*wy - ey, (iy+1)*wy - ey); the last tile
    // loads from ly_last and writes [oy0_last, ny) (a single tile: from -D-ey,
    // writes [0, ny)).  ey puts y = 0 on the last row of a thread's block and
    // ly_last puts y = ny-1 on the first row, so y-shell rows never share a
    // thread with interior rows (their threads copy: coefficients (1, 0)).
    int tiles_y, ey, ly_last, oy0_last;
    int zchunk;        // > 0: segments also end at multiples of zchunk output planes of a
                       // tile (3D blocks: the ablation ladder's 4D bar); 0: z-runs as split
    int ring;          // TMA ring slots (<= ST7_RING_MAX); ring - 2 planes are prefetched ahead
    int pdl;           // host side: launch with programmatic dependent launch
    double alpha, beta;
    int split[ST7_MAX_GRID + 1];   // CTA b owns work items [split[b], split[b+1]) (host cost model)
};

// ---------------------------------------------------------------------------
// one 16-byte row of a thread's block in one plane
//  * FP32: two natural packed pairs a = (c0, c1), b = (c2, c3); the X sums are
//    swap(a) + (L, c2) and swap(b) + (c1, R) (the swaps are free operand
//    swizzles of FADD2, .F32x2.LO_HI), so an update of a pair is 7 packed
//    sm_100a instructions (FADD2 x4, FMUL2, FFMA2 x2) for 2 points.
//  * FP64: two scalars (no packed DP form).
// ---------------------------------------------------------------------------
//  * FP32 narrow layout (VX = 2): one pair c = (c0, c1) per row; the X sums
//    are (L, R) + swap(c) with L, R shuffled straight into a register pair, so
//    no pair is constructed (the 4-wide layout moves one half per X sum).
template <typename T, int VX = Vec<T>::N> struct Rw;
template <> struct Rw<float, 4> { float2 a, b; };
template <> struct Rw<float, 2> { float2 a; };
template <> struct Rw<double, 2> { double x0, x1; };

__device__ __forceinline__ Rw<float, 4> ld_row(const float* s) {
    const float4 v = *reinterpret_cast<const float4*>(s);
    return Rw<float, 4>{make_float2(v.x, v.y), make_float2(v.z, v.w)};
}
__device__ __forceinline__ Rw<double> ld_row(const double* s) {
    const double2 v = *reinterpret_cast<const double2*>(s);
    return Rw<double>{v.x, v.y};
}
template <int VX, typename T>
__device__ __forceinline__ Rw<T, VX> ld_rowv(const T* s) {
    if constexpr (sizeof(T) == 4 && VX == 2) return Rw<float, 2>{*reinterpret_cast<const float2*>(s)};
    else return ld_row(s);
}
__device__ __forceinline__ void st_row(float* s, const Rw<float, 2>& r) { *reinterpret_cast<float2*>(s) = r.a; }
#ifndef ST7_ST64
#define ST7_ST64 0
#endif
__device__ __forceinline__ void st_row(float* s, const Rw<float>& r) {
#if ST7_ST64   // two 8-byte stores: each packed pair is stored from its own register pair
    reinterpret_cast<float2*>(s)[0] = r.a;
    reinterpret_cast<float2*>(s)[1] = r.b;
#else
    *reinterpret_cast<float4*>(s) = make_float4(r.a.x, r.a.y, r.b.x, r.b.y);
#endif
}
__device__ __forceinline__ void st_row(double* s, const Rw<double>& r) {
    *reinterpret_cast<double2*>(s) = make_double2(r.x0, r.x1);
}

template <typename T, int VY, int VX = Vec<T>::N> struct Bk { Rw<T, VX> r[VY]; };

// Per-lane update coefficients.  A point on the x shell (x = 0 or nx-1) is
// Dirichlet-fixed: it gets (alpha, beta) = (1, 0), so the update returns the
// centre exactly (every neighbour sum is finite); y-shell rows are copied in a
// warp-uniform branch, z-shell planes by the non-steady rounds.
template <typename T, int VX = Vec<T>::N> struct St7Coef;
template <> struct St7Coef<float, 2> {
    float2 alA, beA;               // for the pair c = (c0, c1)
    static __device__ __forceinline__ St7Coef make(float al, float be, uint32_t xfix) {
        return St7Coef{make_float2(xfix & 1 ? 1.f : al, xfix & 2 ? 1.f : al),
                       make_float2(xfix & 1 ? 0.f : be, xfix & 2 ? 0.f : be)};
    }
};
template <> struct St7Coef<float, 4> {
    float2 alA, beA, alB, beB;     // for the pairs a = (c0, c1), b = (c2, c3)
    static __device__ __forceinline__ St7Coef make(float al, float be, uint32_t xfix) {  // xfix bit i: column i fixed
#ifdef ST7_AB_SCALAR   // A/B timing only: ignores the shell (wrong values there)
        xfix = 0u;
#endif
        St7Coef k;
        k.alA = make_float2(xfix & 1 ? 1.f : al, xfix & 2 ? 1.f : al);
        k.beA = make_float2(xfix & 1 ? 0.f : be, xfix & 2 ? 0.f : be);
        k.alB = make_float2(xfix & 4 ? 1.f : al, xfix & 8 ? 1.f : al);
        k.beB = make_float2(xfix & 4 ? 0.f : be, xfix & 8 ? 0.f : be);
        return k;
    }
};
template <> struct St7Coef<double, 2> {
    double al0, be0, al1, be1;
    static __device__ __forceinline__ St7Coef make(double al, double be, uint32_t xfix) {
        return St7Coef{xfix & 1 ? 1.0 : al, xfix & 1 ? 0.0 : be, xfix & 2 ? 1.0 : al, xfix & 2 ? 0.0 : be};
    }
};

// y-shell rows (rowfix bit j) keep their value
template <typename T, int VY, int VX>
__device__ __forceinline__ void fix_rows(Bk<T, VY, VX>& O, const Bk<T, VY, VX>& H, uint32_t rowfix) {
#pragma unroll
    for (int j = 0; j < VY; ++j)
        if (rowfix & (1u << j)) O.r[j] = H.r[j];
}

// X neighbours of the rows' edge points from the adjacent lanes (x0 - 1, x0 + VX)
template <int NTX, int VY>
__device__ __forceinline__ void xshfl(const Bk<float, VY>& H, float (&L)[VY], float (&R)[VY]) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        L[j] = __shfl_up_sync(0xffffffffu, H.r[j].b.y, 1, NTX);
        R[j] = __shfl_down_sync(0xffffffffu, H.r[j].a.x, 1, NTX);
    }
}
template <int NTX, int VY>
__device__ __forceinline__ void xshfl(const Bk<double, VY>& H, double (&L)[VY], double (&R)[VY]) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        L[j] = __shfl_up_sync(0xffffffffu, H.r[j].x1, 1, NTX);
        R[j] = __shfl_down_sync(0xffffffffu, H.r[j].x0, 1, NTX);
    }
}

// Phase A of one level.  fast: A = alpha*H + beta*(((y- + y+) + z-) + (x- + x+))
// exact (oracle order X2): A = (x- + x+) + (y- + y+)   (the z terms come in phase C)
template <int NTX, int VY, bool EXACT>
__device__ __forceinline__ void phaseA(const Bk<float, VY>& Zm, const Bk<float, VY>& H, const Rw<float>& top,
                                       const Rw<float>& bot, const St7Coef<float>& k, Bk<float, VY>& A) {
    float L[VY], R[VY];
    xshfl<NTX, VY>(H, L, R);
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        const Rw<float>& ym = j > 0 ? H.r[j - 1] : top;
        const Rw<float>& yp = j < VY - 1 ? H.r[j + 1] : bot;
        const Rw<float>& c = H.r[j];
        // (c0, c1) -> (L + c1, c0 + c2);  (c2, c3) -> (c1 + c3, c2 + R)
        const float2 sxa = __fadd2_rn(make_float2(c.a.y, c.a.x), make_float2(L[j], c.b.x));
        const float2 sxb = __fadd2_rn(make_float2(c.b.y, c.b.x), make_float2(c.a.y, R[j]));
        const float2 sya = __fadd2_rn(ym.a, yp.a), syb = __fadd2_rn(ym.b, yp.b);
        if (EXACT) {
            A.r[j].a = __fadd2_rn(sxa, sya);
            A.r[j].b = __fadd2_rn(sxb, syb);
        } else {
            const float2 sa = __fadd2_rn(__fadd2_rn(sya, Zm.r[j].a), sxa);
            const float2 sb = __fadd2_rn(__fadd2_rn(syb, Zm.r[j].b), sxb);
            A.r[j].a = __ffma2_rn(k.alA, c.a, __fmul2_rn(k.beA, sa));
            A.r[j].b = __ffma2_rn(k.alB, c.b, __fmul2_rn(k.beB, sb));
        }
    }
}
template <int NTX, int VY, bool EXACT>
__device__ __forceinline__ void phaseA(const Bk<double, VY>& Zm, const Bk<double, VY>& H, const Rw<double>& top,
                                       const Rw<double>& bot, const St7Coef<double>& k, Bk<double, VY>& A) {
    double L[VY], R[VY];
    xshfl<NTX, VY>(H, L, R);
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        const Rw<double>& ym = j > 0 ? H.r[j - 1] : top;
        const Rw<double>& yp = j < VY - 1 ? H.r[j + 1] : bot;
        const Rw<double>& c = H.r[j];
        const double sx0 = __dadd_rn(L[j], c.x1), sx1 = __dadd_rn(c.x0, R[j]);
        const double sy0 = __dadd_rn(ym.x0, yp.x0), sy1 = __dadd_rn(ym.x1, yp.x1);
        if (EXACT) {
            A.r[j].x0 = __dadd_rn(sx0, sy0);
            A.r[j].x1 = __dadd_rn(sx1, sy1);
        } else {
            A.r[j].x0 = __fma_rn(k.al0, c.x0, __dmul_rn(k.be0, __dadd_rn(__dadd_rn(sy0, Zm.r[j].x0), sx0)));
            A.r[j].x1 = __fma_rn(k.al1, c.x1, __dmul_rn(k.be1, __dadd_rn(__dadd_rn(sy1, Zm.r[j].x1), sx1)));
        }
    }
}

// narrow FP32 layout: one pair per row, X sums (L + c1, c0 + R) = (L, R) + swap(c)
template <int NTX, int VY, bool EXACT>
__device__ __forceinline__ void phaseA(const Bk<float, VY, 2>& Zm, const Bk<float, VY, 2>& H, const Rw<float, 2>& top,
                                       const Rw<float, 2>& bot, const St7Coef<float, 2>& k, Bk<float, VY, 2>& A) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        const float2 LR = make_float2(__shfl_up_sync(0xffffffffu, H.r[j].a.y, 1, NTX),
                                      __shfl_down_sync(0xffffffffu, H.r[j].a.x, 1, NTX));
        const Rw<float, 2>& ym = j > 0 ? H.r[j - 1] : top;
        const Rw<float, 2>& yp = j < VY - 1 ? H.r[j + 1] : bot;
        const float2 c = H.r[j].a;
        const float2 sx = __fadd2_rn(LR, make_float2(c.y, c.x));
        const float2 sy = __fadd2_rn(ym.a, yp.a);
        if (EXACT) {
            A.r[j].a = __fadd2_rn(sx, sy);
        } else {
            const float2 s_ = __fadd2_rn(__fadd2_rn(sy, Zm.r[j].a), sx);
            A.r[j].a = __ffma2_rn(k.alA, c, __fmul2_rn(k.beA, s_));
        }
    }
}
template <int VY, bool EXACT>
__device__ __forceinline__ void phaseC(const Bk<float, VY, 2>& A, const Bk<float, VY, 2>& Zm, const Bk<float, VY, 2>& H,
                                       const Bk<float, VY, 2>& F, const St7Coef<float, 2>& k, Bk<float, VY, 2>& O) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        if (EXACT) {
            const float2 sa = __fadd2_rn(A.r[j].a, __fadd2_rn(Zm.r[j].a, F.r[j].a));
            const float2 c = H.r[j].a;
            O.r[j].a = make_float2(__fadd_rn(__fmul_rn(k.alA.x, c.x), __fmul_rn(k.beA.x, sa.x)),
                                   __fadd_rn(__fmul_rn(k.alA.y, c.y), __fmul_rn(k.beA.y, sa.y)));
        } else {
            O.r[j].a = __ffma2_rn(k.beA, F.r[j].a, A.r[j].a);
        }
    }
}

// Phase C of one level: out = A + beta*F (fast), or the oracle's
// alpha*c + beta*(q + (z- + z+)) with every operation rounded (exact)
template <int VY, bool EXACT>
__device__ __forceinline__ void phaseC(const Bk<float, VY>& A, const Bk<float, VY>& Zm, const Bk<float, VY>& H,
                                       const Bk<float, VY>& F, const St7Coef<float>& k, Bk<float, VY>& O) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        if (EXACT) {
            const float2 sa = __fadd2_rn(A.r[j].a, __fadd2_rn(Zm.r[j].a, F.r[j].a));
            const float2 sb = __fadd2_rn(A.r[j].b, __fadd2_rn(Zm.r[j].b, F.r[j].b));
            const Rw<float>& c = H.r[j];
            O.r[j].a = make_float2(__fadd_rn(__fmul_rn(k.alA.x, c.a.x), __fmul_rn(k.beA.x, sa.x)),
                                   __fadd_rn(__fmul_rn(k.alA.y, c.a.y), __fmul_rn(k.beA.y, sa.y)));
            O.r[j].b = make_float2(__fadd_rn(__fmul_rn(k.alB.x, c.b.x), __fmul_rn(k.beB.x, sb.x)),
                                   __fadd_rn(__fmul_rn(k.alB.y, c.b.y), __fmul_rn(k.beB.y, sb.y)));
        } else {
            O.r[j].a = __ffma2_rn(k.beA, F.r[j].a, A.r[j].a);
            O.r[j].b = __ffma2_rn(k.beB, F.r[j].b, A.r[j].b);
        }
    }
}
template <int VY, bool EXACT>
__device__ __forceinline__ void phaseC(const Bk<double, VY>& A, const Bk<double, VY>& Zm, const Bk<double, VY>& H,
                                       const Bk<double, VY>& F, const St7Coef<double>& k, Bk<double, VY>& O) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        if (EXACT) {
            const double s0 = __dadd_rn(A.r[j].x0, __dadd_rn(Zm.r[j].x0, F.r[j].x0));
            const double s1 = __dadd_rn(A.r[j].x1, __dadd_rn(Zm.r[j].x1, F.r[j].x1));
            O.r[j].x0 = __dadd_rn(__dmul_rn(k.al0, H.r[j].x0), __dmul_rn(k.be0, s0));
            O.r[j].x1 = __dadd_rn(__dmul_rn(k.al1, H.r[j].x1), __dmul_rn(k.be1, s1));
        } else {
            O.r[j].x0 = __fma_rn(k.be0, F.r[j].x0, A.r[j].x0);
            O.r[j].x1 = __fma_rn(k.be1, F.r[j].x1, A.r[j].x1);
        }
    }
}

// XY placement of tile `tile` (row-major over tiles_x): loaded box corner
// (Lx, Ly) and written region [ox0, ox1) x [oy0, oy1)
struct St7Tile { int Lx, Ly, ox0, ox1, oy0, oy1; };
__device__ __forceinline__ St7Tile st7_tile(const St7Params& p, int tile, int D) {
    St7Tile t;
    const int ix = tile % p.tiles_x, iy = tile / p.tiles_x;
    t.ox0 = ix * p.wx;
    t.ox1 = min(t.ox0 + p.wx, p.nx);
    t.Lx = t.ox0 - p.hx;
    if (p.tiles_y == 1) {
        t.Ly = -D - p.ey; t.oy0 = 0; t.oy1 = p.ny;
    } else if (iy == p.tiles_y - 1) {
        t.Ly = p.ly_last; t.oy0 = p.oy0_last; t.oy1 = p.ny;
    } else {
        t.oy0 = max(iy * p.wy - p.ey, 0);
        t.oy1 = min((iy + 1) * p.wy - p.ey, p.ny);
        t.Ly = iy * p.wy - D - p.ey;
    }
    return t;
}

// NT threads per CTA, MINB CTAs per SM (register cap 65536 / (NT * MINB));
// SPLIT: two-phase rounds (false: level by level, the ablation ladder's
// pre-ILP bar)
// VXK: points per thread row (0: one 16-byte vector, 4 FP32 / 2 FP64; 2 for
// FP32: the narrow layout, 32 threads across the 64-point tile row)
// compile-time loop: f(integral_constant<int, I>) for I = B..E-1
template <int B, int E, typename F>
__device__ __forceinline__ void static_for(F&& f) {
    if constexpr (B < E) {
        f(std::integral_constant<int, B>{});
        static_for<B + 1, E>(f);
    }
}

#ifdef ST7_TRACE
// A/B diagnostics build only (-DST7_TRACE): per CTA globaltimer stamps
// [entry, after pdl_wait, (segment start, first steady round, steady end) x 3,
// end, segment count, first 3 segment lengths (16 bits each)]
static __device__ unsigned long long st7_trace_buf[ST7_MAX_GRID][16];
// first 16 rounds of segment 0: [round][0] plane landed (after mbar_wait), [1] round end
static __device__ unsigned long long st7_trace_rnd[ST7_MAX_GRID][16][2];
static __device__ unsigned long long st7_trace_iss[ST7_MAX_GRID][16];   // segment 0: issue time of load k
__device__ __forceinline__ unsigned long long st7_gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#define ST7_STAMP(i, v) do { if (threadIdx.x == 0) st7_trace_buf[blockIdx.x][i] = (v); } while (0)
#else
#define ST7_STAMP(i, v) do { } while (0)
#endif

template <typename T, int D, int NTX, int VY, bool EXACT, int NT, int MINB, bool SPLIT = true, int VXK = 0>
__global__ void __launch_bounds__(NT, MINB)
st7_35d_kernel(const __grid_constant__ CUtensorMap tmap, const St7Params p) {
    constexpr int VX = VXK ? VXK : (sizeof(T) == 4 ? 4 : 2);
    constexpr int TX = NTX * VX;
    const int NTH = blockDim.x;         // threads (<= NT): NTY rows of NTX threads
    const int NTY = NTH / NTX;
    const int TY = NTY * VY;
    using V = typename std::conditional<VX * sizeof(T) == 16, typename std::conditional<sizeof(T) == 4, float4, double2>::type,
                                        float2>::type;   // one exchanged row
    using B = Bk<T, VY, VX>;
    using RW = Rw<T, VX>;

    extern __shared__ __align__(128) unsigned char smem_raw[];
#ifdef ST7_TRACE
    ST7_STAMP(0, st7_gtime());
    int nseg_tr = 0;
#endif
    const int tid = threadIdx.x;
    const int tx = tid % NTX;
    const int ty = tid / NTX;
    const T al = T(p.alpha), be = T(p.beta);

    // ring of RING level-0 plane slots: round r reads planes r-1 (Y-edge rows
    // of level 1's centre) and r; PF = RING-2 planes are in flight
    const int RING = p.ring, PF = p.ring - 2;
    const int slot_elems = TX * TY;
    const uint32_t slot_bytes = (uint32_t)(slot_elems * sizeof(T));
    T* ring = reinterpret_cast<T*>(smem_raw);                      // [RING][TY][TX]
    // row exchange [level 1..D-1][parity][N row / S row][NT] (16-byte rows)
    V* xbuf = reinterpret_cast<V*>(ring + RING * slot_elems);
    uint64_t* bars = reinterpret_cast<uint64_t*>(xbuf + (D > 1 ? (D - 1) * 4 * NTH : 0));

    // zero the ring once: a fixed (shell) point of a plane may sit next to a
    // never-loaded slot row; every value that is read must be finite
    for (int i = tid; i < RING * slot_elems * (int)sizeof(T) / 16; i += NTH)
        reinterpret_cast<float4*>(ring)[i] = make_float4(0.f, 0.f, 0.f, 0.f);
    fence_proxy_async();   // generic-proxy writes before the first TMA (async proxy) writes
    if (tid == 0) {
        prefetch_tensormap(&tmap);
        for (int s = 0; s < RING; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
    }
    __syncthreads();
    // PDL: the setup above overlapped the previous sweep's tail; its output
    // (this sweep's input) and its reads of our output buffer are complete here
    pdl_trigger();
    pdl_wait();
#ifdef ST7_TRACE
    ST7_STAMP(1, st7_gtime());
#endif

    // register window: pl[k][*] holds planes of level k (0..D-1), three slots
    // rotating with the round (z-1, z, new); level 0 is loaded from the ring
    B pl[D][3];
#pragma unroll
    for (int l = 0; l < D; ++l)
#pragma unroll
        for (int k = 0; k < 3; ++k)
#pragma unroll
            for (int j = 0; j < VY; ++j) pl[l][k].r[j] = RW{};

    const int nzo = p.zb - p.za;
    int item = p.split[blockIdx.x];
    const int item_end = p.split[blockIdx.x + 1];
    const int zmin = max(0, -p.zbase);
    const int zmax = min(p.nzb - 1, p.nzg - 1 - p.zbase);
    const int my_off = (VY * ty) * TX + VX * tx;                   // my first row in a plane
    const int top_off = max(VY * ty - 1, 0) * TX + VX * tx;         // row above my block
    const int bot_off = min(VY * ty + VY, TY - 1) * TX + VX * tx;   // row below my block
    const int tyu = max(ty - 1, 0), tyd = min(ty + 1, NTY - 1);
    const size_t plane = (size_t)p.nx * p.ny;
    uint32_t nload = 0;       // ring sequence number of the next segment's first plane

    // segment = the part of this CTA's work range inside one tile: output
    // planes [za, zb), level-0 planes [rl0, rl1] of tile `tile`
    struct Seg { int tile, za, zb, rl0, rl1; };
    auto seg_at = [&](int it) {
        Seg g;
        g.tile = it / nzo;
        int seg_end = min(item_end, (g.tile + 1) * nzo);
        if (p.zchunk > 0) seg_end = min(seg_end, it + (p.zchunk - (it - g.tile * nzo) % p.zchunk));
        g.za = p.za + (it - g.tile * nzo);
        g.zb = p.za + (seg_end - g.tile * nzo);
        g.rl0 = max(g.za - D, zmin);
        g.rl1 = min(g.zb - 1 + D, zmax);
        return g;
    };
    int pre = 0;   // loads of the NEXT segment issued during this one's epilog (thread 0 only)

    while (item < item_end) {
        const Seg sg = seg_at(item);
#ifdef ST7_TRACE
        if (nseg_tr == 0) {
            unsigned smid;
            asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
            ST7_STAMP(15, (unsigned long long)sg.tile | ((unsigned long long)smid << 16) |
                              ((unsigned long long)sg.za << 32));
        }
        if (nseg_tr < 3) ST7_STAMP(2 + 3 * nseg_tr, st7_gtime());
        if (nseg_tr < 3) ST7_STAMP(14, (nseg_tr ? st7_trace_buf[blockIdx.x][14] : 0ull) |
                                           ((unsigned long long)(sg.zb - sg.za) << (16 * nseg_tr)));
        ++nseg_tr;
#endif
        const int za = sg.za, zb = sg.zb, rl0 = sg.rl0, rl1 = sg.rl1;
        item += zb - za;
        const bool has_next = item < item_end;
        const Seg nx = seg_at(has_next ? item : item - 1);
        const St7Tile tl = st7_tile(p, sg.tile, D);
        const St7Tile tn = st7_tile(p, nx.tile, D);

        const int xg0 = tl.Lx + VX * tx;
        uint32_t xfix = 0, rowfix = 0, rowout = 0, rowmask = 0;
#pragma unroll
        for (int i = 0; i < VX; ++i)
            if (xg0 + i == 0 || xg0 + i == p.nx - 1) xfix |= 1u << i;
#pragma unroll
        for (int j = 0; j < VY; ++j) {
            const int yg = tl.Ly + VY * ty + j;
            if (yg >= tl.oy0 && yg < tl.oy1) rowmask |= 1u << j;
            if (yg == 0 || yg == p.ny - 1) rowfix |= 1u << j;
            if (yg < 0 || yg >= p.ny) rowout |= 1u << j;
        }
        // a thread whose rows are all y-shell or outside the grid copies (the
        // planner's y placement makes this the case for every y-shell row);
        // otherwise its warp takes the checked round body with row fix-ups
        const bool allfix = rowfix != 0 && (rowfix | rowout) == (1u << VY) - 1;
        const bool yslow = __any_sync(0xffffffffu, rowfix != 0 && !allfix);   // warp-uniform
        if (!(xg0 >= tl.ox0 && xg0 < tl.ox1)) rowmask = 0;    // vectors are all-in or all-out in x
        const St7Coef<T, VX> kc = St7Coef<T, VX>::make(al, be, allfix ? 0xFu : xfix);

        const int r0 = rl0, r1 = zb - 1 + D;
        // steady rounds: every level active, no z-shell plane among the computed ones
        const int rs0 = max(max(za + D, zmin + D), -p.zbase + D + 1);
        const int rs1 = min(min(zb - 1 + D, zmax + 1), min(rl1, p.nzg - 1 - p.zbase));
        T* pout = reinterpret_cast<T*>(p.out) + xg0 + (size_t)(tl.Ly + VY * ty) * p.nx +
                  (long long)(r0 - D) * (long long)plane;   // level D at round r: plane r - D
        const uint32_t kbase = nload;
        if (tid == 0) {
            for (int q = rl0 + pre; q <= min(rl0 + PF - 1, rl1); ++q) {
                const uint32_t k = (kbase + (q - rl0)) % RING;
                mbar_arrive_expect_tx(&bars[k], slot_bytes);
                tma_load_3d(ring + k * slot_elems, &tmap, &bars[k], tl.Lx, tl.Ly, q);
#ifdef ST7_TRACE
                if (nseg_tr == 1 && q - rl0 < 16) st7_trace_iss[blockIdx.x][q - rl0] = st7_gtime();
#endif
            }
            pre = 0;
        }
        nload = kbase + (uint32_t)max(0, rl1 - rl0 + 1);
        // ring slot / parity of plane r (sequence kbase + r - rl0), of r + PF and of r - 1
        uint32_t slot_r = kbase % RING, par_r = (kbase / RING) & 1;
        uint32_t slot_f = (kbase + PF) % RING;
        uint32_t slot_m1 = (slot_r + RING - 1) % RING;

        // NACTc: -1 = checked round; n >= 0 = unchecked round with levels 1..n
        // active (n = D: a steady round; n < D: a prolog round, no output)
        auto round = [&](auto PHc, auto NACTc, int r) {
            constexpr int PH = decltype(PHc)::value;
            constexpr int NACT = decltype(NACTc)::value;
            constexpr bool STEADY = NACT >= 0;
            constexpr int PREV = PH % 3, CUR = (PH + 1) % 3, NEW = (PH + 2) % 3;
            const int rpar = r & 1;
            // load plane r + PF into the slot plane r-2 left (free since round r-1's barrier)
            if (tid == 0) {
                if (r + PF <= rl1) {
                    mbar_arrive_expect_tx(&bars[slot_f], slot_bytes);
                    tma_load_3d(ring + slot_f * slot_elems, &tmap, &bars[slot_f], tl.Lx, tl.Ly, r + PF);
#ifdef ST7_TRACE
                    if (nseg_tr == 1 && r + PF - rl0 < 16) st7_trace_iss[blockIdx.x][r + PF - rl0] = st7_gtime();
#endif
                } else if (has_next && pre < PF && pre == r + PF - rl1 - 1 && nx.rl0 + pre <= nx.rl1) {
                    // sequence kbase + (r + PF - rl0) is the next segment's plane rl0' + pre
                    mbar_arrive_expect_tx(&bars[slot_f], slot_bytes);
                    tma_load_3d(ring + slot_f * slot_elems, &tmap, &bars[slot_f], tn.Lx, tn.Ly, nx.rl0 + pre);
                    ++pre;
                }
            }
            // Non-steady rounds (prolog, epilog, z-shell planes, warps with an
            // unaligned y-shell row) run the same body plus checks: a level whose
            // plane lies outside its range is skipped (warp-uniform); a level on a
            // z-shell plane copies its centre (fixed boundary); the final level
            // stores only output planes.
            bool zf[D + 1], act[D + 1];
#pragma unroll
            for (int l = 1; l <= D; ++l) {
                zf[l] = false;
                act[l] = !STEADY || l <= NACT;
                if (!STEADY) {   // level l computes plane r - l: inside its range, or skipped
                    const int zg = p.zbase + r - l;
                    zf[l] = zg == 0 || zg == p.nzg - 1;
                    const int lo = max(za - (D - l), zmin), hi = min(zb - 1 + (D - l), zmax);
                    act[l] = r - l >= lo && r - l <= hi;
                }
            }
            // ---- phase A: in-plane part of every level (no dependence on this round's planes);
            // fast: the result replaces the dead z-1 plane of the level's input
            B acc[EXACT ? D + 1 : 1];
            auto level_A = [&](int l) {
                const int k = l - 1;
                RW top, bot;
                if (l == 1) {   // level-0 neighbour rows of plane r-1 straight from the ring
                    const T* sl = ring + slot_m1 * slot_elems;
                    top = ld_rowv<VX>(sl + top_off);
                    bot = ld_rowv<VX>(sl + bot_off);
                } else {        // rows the blocks above / below exchanged in round r-1
                    const V* xb = xbuf + ((l - 2) * 4 + (rpar ^ (l & 1)) * 2) * NTH;   // by level l-1 in round r-1
                    top = ld_rowv<VX>(reinterpret_cast<const T*>(xb + NTH + tyu * NTX + tx));
                    bot = ld_rowv<VX>(reinterpret_cast<const T*>(xb + tyd * NTX + tx));
                }
                phaseA<NTX, VY, EXACT>(pl[k][PREV], pl[k][CUR], top, bot, kc, EXACT ? acc[EXACT ? l : 0] : pl[k][PREV]);
            };
            // ---- level 0, plane r: landed in the ring -> my rows into the register window
            auto load0 = [&]() {
                if (STEADY || r <= rl1) {
                    mbar_wait(&bars[slot_r], par_r);
#ifdef ST7_TRACE
                    if (tid == 0 && nseg_tr == 1 && r - r0 < 16) st7_trace_rnd[blockIdx.x][r - r0][0] = st7_gtime();
#endif
                    const T* s0 = ring + slot_r * slot_elems + my_off;
#pragma unroll
                    for (int j = 0; j < VY; ++j) pl[0][NEW].r[j] = ld_rowv<VX>(s0 + j * TX);
                }
            };
            // ---- phase C: the z+1 term along the level chain
            auto level_C = [&](int l) {
                const int k = l - 1;
                B out;
                phaseC<VY, EXACT>(EXACT ? acc[EXACT ? l : 0] : pl[k][PREV], pl[k][PREV], pl[k][CUR], pl[k][NEW], kc, out);
                if (!STEADY) {   // unaligned y-shell rows and z-shell planes: fixed
                    if (yslow) fix_rows(out, pl[k][CUR], rowfix);
                    if (zf[l]) out = pl[k][CUR];
                }
                if (l < D) {
                    pl[l < D ? l : 0][NEW] = out;
                    T* xb = reinterpret_cast<T*>(xbuf + ((l - 1) * 4 + (rpar ^ (l & 1)) * 2) * NTH + tid);
                    st_row(xb, out.r[0]);
                    st_row(xb + NTH * VX, out.r[VY - 1]);
                } else if (STEADY || (r - D >= za && r - D < zb)) {
#pragma unroll
                    for (int j = 0; j < VY; ++j)
                        if (rowmask & (1u << j)) st_row(pout + j * p.nx, out.r[j]);
                }
            };
            // (a skipped level's planes are never read: the level above is outside
            // its range in the rounds that would read them)
            if (SPLIT) {   // all in-plane parts first, then the z+1 chain
#pragma unroll
                for (int l = 1; l <= D; ++l)
                    if (act[l]) level_A(l);
                load0();
#pragma unroll
                for (int l = 1; l <= D; ++l)
                    if (act[l]) level_C(l);
            } else {           // level by level
                load0();
#pragma unroll
                for (int l = 1; l <= D; ++l)
                    if (act[l]) { level_A(l); level_C(l); }
            }
            __syncthreads();
#ifdef ST7_TRACE
            if (tid == 0 && nseg_tr == 1 && r - r0 < 16) st7_trace_rnd[blockIdx.x][r - r0][1] = st7_gtime();
#endif
            pout += plane;
            slot_m1 = slot_r;
            if (++slot_r == (uint32_t)RING) { slot_r = 0; par_r ^= 1; }
            if (++slot_f == (uint32_t)RING) slot_f = 0;
        };
        using I0 = std::integral_constant<int, 0>;
        using I1 = std::integral_constant<int, 1>;
        using I2 = std::integral_constant<int, 2>;
        using ND = std::integral_constant<int, D>;
        using NCHK = std::integral_constant<int, -1>;
        // Steady rounds (every level active, no z-shell plane, no unaligned
        // y-shell row in the warp) run as
        // back-to-back phase triples without any check; the other rounds take
        // the checked body.  ph = (r - r0) mod 3 selects the register slots.
        const int rs1x = rs1;
        int r = r0, ph = 0;
        // prolog of a segment away from the z faces: round k = 0..2D-1 runs
        // levels 1..k/2 (level l starts at plane za - D + l in round 2l) as
        // compile-time rounds without checks; its register phase starts at
        // (-2D) mod 3 so that the steady triples follow at phase 0
        if (!yslow && r0 == za - D && r0 + 2 * D == rs0 && p.zbase + za - D >= 1 &&
            p.zbase + za + D < p.nzg - 1 && za + D - 1 <= rl1) {
            constexpr int PH0 = (3 - (2 * D) % 3) % 3;
            static_for<0, 2 * D>([&](auto K) {
                constexpr int k = decltype(K)::value;
                round(std::integral_constant<int, (PH0 + k) % 3>{}, std::integral_constant<int, k / 2>{}, r0 + k);
            });
            r = r0 + 2 * D;
        }
        while (r <= r1) {
            if (ph == 0 && !yslow && r >= rs0 && r + 2 <= rs1x) {
#ifdef ST7_TRACE
                if (nseg_tr <= 3) ST7_STAMP(3 * nseg_tr, st7_gtime());
#endif
                do {
                    round(I0{}, ND{}, r);
                    round(I1{}, ND{}, r + 1);
                    round(I2{}, ND{}, r + 2);
                    r += 3;
                } while (r + 2 <= rs1x);
#ifdef ST7_TRACE
                if (nseg_tr <= 3) ST7_STAMP(3 * nseg_tr + 1, st7_gtime());
#endif
                continue;
            }
            if (ph == 0) round(I0{}, NCHK{}, r);
            else if (ph == 1) round(I1{}, NCHK{}, r);
            else round(I2{}, NCHK{}, r);
            ++r;
            ph = ph == 2 ? 0 : ph + 1;
        }
    }
#ifdef ST7_TRACE
    ST7_STAMP(12, st7_gtime());
    ST7_STAMP(13, (unsigned long long)nseg_tr);
#endif
}

}  // namespace st35d
