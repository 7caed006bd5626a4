// st7_kernel.cuh — 3.5D-blocked 7-point Jacobi sweep for sm_100a.
//
// Method (§V): an XY sub-plane (tile) is streamed along Z (2.5D
// blocking) while dim_T time levels are kept on chip (1D temporal
// blocking); only level 0 is read from HBM and only level dim_T is
// written.  Stencil: P:111, boundary fixed (X1).
//
// B200 mapping:
//  * persistent CTAs; each takes an equal share of (tile, z) work items in
//    tile-major order (flexible load balance);
//  * level 0: TMA bulk-tensor loads of the (TX x TY) plane box into a 4-slot
//    shared-memory ring with mbarrier completion, prefetched 2 planes ahead;
//  * every thread owns a VX x VY block of the tile (VX = one 16-byte vector)
//    at all levels, and keeps, for every level, the planes z-1, z, z+1 of its
//    own points in REGISTERS (Z neighbours in registers; the 3 register slots
//    rotate with the round, the round loop is unrolled by 3 so no moves);
//  * X neighbours at the thread-block edge come from the neighbouring lane by
//    warp shuffle; Y neighbours at the block edge from the thread above/below
//    through a small shared-memory row exchange (2 vectors per thread per
//    level, double-buffered by plane parity);
//  * lag 1 per level: level l at round r computes plane r-l; its z+1 input is
//    the thread's own register value produced earlier in the same round, its
//    in-plane neighbours were exchanged in round r-1, so ONE __syncthreads
//    per round suffices (the paper needs lag 2R and 2R+2 buffers per level
//    for the same concurrency, because its planes live in cache);
//  * the final level is written with 128-bit stores of the valid region only.
#pragma once
#include <type_traits>
#include "common.cuh"

#ifndef ST_ZLAST
#define ST_ZLAST 0
#endif
#ifndef ST7_DBG
#define ST7_DBG 0
#endif
#ifndef ST7_L0REG
#define ST7_L0REG 1
#endif
#ifndef ST7_LOOKAHEAD
#define ST7_LOOKAHEAD 0
#endif
#ifndef ST7_PROF
#define ST7_PROF 0
#endif
#ifndef ST7_STEADY_LOOP
#define ST7_STEADY_LOOP (sizeof(T) == 8)   // measured: +3% FP64; FP32 D=4 spills with it
#endif

namespace st35d {

constexpr int ST7_MAX_GRID = 160;   // >= SM count (148 on B200); one persistent CTA per SM

struct St7Params {
    void* out;
    int nx, ny;        // plane extent
    int nzb;           // planes in the local buffer (tensor map extent)
    int zbase;         // global z of local plane 0
    int nzg;           // global nz
    int za, zb;        // local output planes [za, zb)
    int tiles_x, ntiles;
    int wx, wy;        // written region per tile
    int hx;            // x halo (>= D, multiple of VX)
    long long work;    // ntiles * (zb - za)
    int ring;          // TMA ring slots (<= ST7_RING_MAX); ring - 2 planes are prefetched ahead
    int dbg;           // tuning only: bit 0 = stream planes without computing levels
    double alpha, beta;
    int split[ST7_MAX_GRID + 1];   // CTA b owns work items [split[b], split[b+1]) (host cost model)
    unsigned long long* prof;      // ST7_PROF builds only: per-warp phase clocks [cta][warp][10]
};

constexpr int ST7_RING_MAX = 12;

// ---------------------------------------------------------------------------
// One thread's register block of one plane: VY rows x VX columns.
//  * FP32 (VX = 4): each row is held as two natural packed pairs a = (c0, c1),
//    b = (c2, c3) (16-byte rows load, exchange and store with no moves); the X
//    sums are swap(a) + (L, c2) and swap(b) + (c1, R) with L, R shuffled from
//    the neighbouring lanes, and every 7-point update of a pair is 7 packed
//    sm_100a instructions (FADD2 x5, FMUL2, FFMA2) for 2 points.
//  * FP64 (VX = 2): plain scalars (the DP pipe is half rate; no packed form).
// The bit-exact build uses the oracle's order (X2): ((x- + x+) + (y- + y+)) +
// (z- + z+), then alpha*c + beta*s with scalar __fmul_rn / __fadd_rn; the
// tolerance build adds the shuffled X sum last and fuses the final combine.
// ---------------------------------------------------------------------------
template <typename T, int VY> struct Blk;
template <typename T> struct Row;

template <> struct Row<float> { float2 a, b; };
template <> struct Row<double> { double v[2]; };

template <int VY> struct Blk<float, VY> {
    float2 a[VY], b[VY];   // natural pairs: a = (c0, c1), b = (c2, c3): 16-byte rows load/store with no moves
    __device__ __forceinline__ void load_nat(int j, const float* s) {   // smem, natural order
        const float4 v = *reinterpret_cast<const float4*>(s);
        a[j] = make_float2(v.x, v.y);
        b[j] = make_float2(v.z, v.w);
    }
    __device__ __forceinline__ void store_x(int j, float4* s) const {   // exchange row
        *s = make_float4(a[j].x, a[j].y, b[j].x, b[j].y);
    }
    __device__ __forceinline__ void store_global(int j, float* g) const {  // plain store: predicable
        *reinterpret_cast<float4*>(g) = make_float4(a[j].x, a[j].y, b[j].x, b[j].y);
    }
};
template <int VY> struct Blk<double, VY> {
    double v[VY][2];
    __device__ __forceinline__ void load_nat(int j, const double* s) {
        const double2 t = *reinterpret_cast<const double2*>(s);
        v[j][0] = t.x; v[j][1] = t.y;
    }
    __device__ __forceinline__ void store_x(int j, double2* s) const { *s = make_double2(v[j][0], v[j][1]); }
    __device__ __forceinline__ void store_global(int j, double* g) const {
        *reinterpret_cast<double2*>(g) = make_double2(v[j][0], v[j][1]);
    }
};

__device__ __forceinline__ Row<float> row_nat(const float* s) {
    const float4 v = *reinterpret_cast<const float4*>(s);
    return Row<float>{make_float2(v.x, v.y), make_float2(v.z, v.w)};
}
__device__ __forceinline__ Row<float> row_x(const float4* s) {
    const float4 v = *s;
    return Row<float>{make_float2(v.x, v.y), make_float2(v.z, v.w)};
}
__device__ __forceinline__ Row<double> row_nat(const double* s) {
    const double2 v = *reinterpret_cast<const double2*>(s);
    return Row<double>{{v.x, v.y}};
}
__device__ __forceinline__ Row<double> row_x(const double2* s) {
    const double2 v = *s;
    return Row<double>{{v.x, v.y}};
}

// Bit-exact combine alpha*c + beta*s: ptxas 12.9 fuses mul.rn.f32x2 followed by
// add.rn.f32x2 into FFMA2 even with -fmad=false, so the exact build does the
// final combine with scalar __fmul_rn / __fadd_rn (which are never fused).
__device__ __forceinline__ float2 combine_exact(float al, float2 c, float be, float2 s) {
    return make_float2(__fadd_rn(__fmul_rn(al, c.x), __fmul_rn(be, s.x)),
                       __fadd_rn(__fmul_rn(al, c.y), __fmul_rn(be, s.y)));
}

// Per-thread update coefficients.  A point on the x shell (x = 0 or nx-1)
// is Dirichlet-fixed: it gets alpha = 1, beta = 0, so alpha*c + beta*s == c
// exactly (s is always finite here: every neighbour is loaded data or a
// finite combination of it).  Rows on the y shell are copied in a rare
// warp-uniform branch; whole z-shell planes use Coef::fixed().
template <typename T> struct Coef;
template <> struct Coef<float> {
    float2 alA, beA, alB, beB;     // for the pairs a = (c0, c1), b = (c2, c3)
    static __device__ __forceinline__ Coef fixed() {
        return Coef{make_float2(1.f, 1.f), make_float2(0.f, 0.f), make_float2(1.f, 1.f), make_float2(0.f, 0.f)};
    }
    static __device__ __forceinline__ Coef make(float al, float be, uint32_t xfix) {  // xfix bit i: column i fixed
        Coef k;
        k.alA = make_float2(xfix & 1 ? 1.f : al, xfix & 2 ? 1.f : al);
        k.beA = make_float2(xfix & 1 ? 0.f : be, xfix & 2 ? 0.f : be);
        k.alB = make_float2(xfix & 4 ? 1.f : al, xfix & 8 ? 1.f : al);
        k.beB = make_float2(xfix & 4 ? 0.f : be, xfix & 8 ? 0.f : be);
        return k;
    }
    // field-wise select (a ?: on the structs would take their addresses -> local memory)
    static __device__ __forceinline__ Coef sel(bool f, const Coef& x, const Coef& y) {
        return Coef{f ? x.alA : y.alA, f ? x.beA : y.beA, f ? x.alB : y.alB, f ? x.beB : y.beB};
    }
};
template <> struct Coef<double> {
    double al[2], be[2];
    static __device__ __forceinline__ Coef fixed() { return Coef{{1.0, 1.0}, {0.0, 0.0}}; }
    static __device__ __forceinline__ Coef make(double al, double be, uint32_t xfix) {
        return Coef{{xfix & 1 ? 1.0 : al, xfix & 2 ? 1.0 : al}, {xfix & 1 ? 0.0 : be, xfix & 2 ? 0.0 : be}};
    }
    static __device__ __forceinline__ Coef sel(bool f, const Coef& x, const Coef& y) {
        return Coef{{f ? x.al[0] : y.al[0], f ? x.al[1] : y.al[1]}, {f ? x.be[0] : y.be[0], f ? x.be[1] : y.be[1]}};
    }
};

// X neighbours of a block's rows from the neighbouring lanes (x0 - 1 and x0 + VX):
// issued one level ahead by the kernel so the shuffle latency overlaps a level
template <typename T, int VY> struct XN { T l[VY], r[VY]; };
template <int NTX, int VY>
__device__ __forceinline__ XN<float, VY> xshuf(const Blk<float, VY>& C) {
    XN<float, VY> x;
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        x.l[j] = __shfl_up_sync(0xffffffffu, C.b[j].y, 1, NTX);
        x.r[j] = __shfl_down_sync(0xffffffffu, C.a[j].x, 1, NTX);
    }
    return x;
}
template <int NTX, int VY>
__device__ __forceinline__ XN<double, VY> xshuf(const Blk<double, VY>& C) {
    XN<double, VY> x;
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        x.l[j] = __shfl_up_sync(0xffffffffu, C.v[j][1], 1, NTX);
        x.r[j] = __shfl_down_sync(0xffffffffu, C.v[j][0], 1, NTX);
    }
    return x;
}

// one level of the sweep for one thread's block: R = stencil(ZM, C, ZP)
// (PRE: X neighbours pre-shuffled in xn; otherwise shuffled here, row by row)
template <int NTX, int VY, bool EXACT, bool PRE = true>
__device__ __forceinline__ void st7_level(const Blk<float, VY>& ZM, const Blk<float, VY>& C,
                                          const Blk<float, VY>& ZP, const XN<float, VY>& xn, const Row<float>& top,
                                          const Row<float>& bot, const Coef<float>& k, bool yslow,
                                          uint32_t rowfix, Blk<float, VY>& R) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        const float left = PRE ? xn.l[j] : __shfl_up_sync(0xffffffffu, C.b[j].y, 1, NTX);     // x0 - 1
        const float right = PRE ? xn.r[j] : __shfl_down_sync(0xffffffffu, C.a[j].x, 1, NTX);  // x0 + 4
        const float2 yma = j > 0 ? C.a[j - 1] : top.a, ypa = j < VY - 1 ? C.a[j + 1] : bot.a;
        const float2 ymb = j > 0 ? C.b[j - 1] : top.b, ypb = j < VY - 1 ? C.b[j + 1] : bot.b;
        // X sums (x-1 + x+1): (c0, c1) -> (c1 + L, c0 + c2) = swap(a) + (L, c2);
        // (c2, c3) -> (c3 + c1, c2 + R) = swap(b) + (c1, R).  The swapped pairs are
        // operand swizzles (.LO_HI), so only one half of each constructed pair moves.
        const float2 sxa = __fadd2_rn(make_float2(C.a[j].y, C.a[j].x), make_float2(left, C.b[j].x));
        const float2 sxb = __fadd2_rn(make_float2(C.b[j].y, C.b[j].x), make_float2(C.a[j].y, right));
        float2 sa, sb;
        if (EXACT) {   // oracle order (X2)
            sa = __fadd2_rn(__fadd2_rn(sxa, __fadd2_rn(yma, ypa)), __fadd2_rn(ZM.a[j], ZP.a[j]));
            sb = __fadd2_rn(__fadd2_rn(sxb, __fadd2_rn(ymb, ypb)), __fadd2_rn(ZM.b[j], ZP.b[j]));
        } else if (ST_ZLAST) {
            // tolerance build: the z+1 plane (produced by the previous level in this
            // same round) enters last, by FMA, so consecutive levels overlap:
            // R = beta*zp + (alpha*c + beta*((y + x) + zm)) -- still 7 packed ops
            sa = __fadd2_rn(__fadd2_rn(__fadd2_rn(yma, ypa), sxa), ZM.a[j]);
            sb = __fadd2_rn(__fadd2_rn(__fadd2_rn(ymb, ypb), sxb), ZM.b[j]);
        } else {       // shuffled X terms last: the y/z sums overlap the shuffle latency
            sa = __fadd2_rn(__fadd2_rn(__fadd2_rn(yma, ypa), __fadd2_rn(ZM.a[j], ZP.a[j])), sxa);
            sb = __fadd2_rn(__fadd2_rn(__fadd2_rn(ymb, ypb), __fadd2_rn(ZM.b[j], ZP.b[j])), sxb);
        }
        if (!EXACT && ST_ZLAST) {
            R.a[j] = __ffma2_rn(k.beA, ZP.a[j], __ffma2_rn(k.alA, C.a[j], __fmul2_rn(k.beA, sa)));
            R.b[j] = __ffma2_rn(k.beB, ZP.b[j], __ffma2_rn(k.alB, C.b[j], __fmul2_rn(k.beB, sb)));
        } else if (EXACT) {
            R.a[j] = make_float2(__fadd_rn(__fmul_rn(k.alA.x, C.a[j].x), __fmul_rn(k.beA.x, sa.x)),
                                 __fadd_rn(__fmul_rn(k.alA.y, C.a[j].y), __fmul_rn(k.beA.y, sa.y)));
            R.b[j] = make_float2(__fadd_rn(__fmul_rn(k.alB.x, C.b[j].x), __fmul_rn(k.beB.x, sb.x)),
                                 __fadd_rn(__fmul_rn(k.alB.y, C.b[j].y), __fmul_rn(k.beB.y, sb.y)));
        } else {
            R.a[j] = __ffma2_rn(k.alA, C.a[j], __fmul2_rn(k.beA, sa));
            R.b[j] = __ffma2_rn(k.alB, C.b[j], __fmul2_rn(k.beB, sb));
        }
    }
    if (yslow) {  // warp-uniform: only warps holding a y-shell row
#pragma unroll
        for (int j = 0; j < VY; ++j)
            if (rowfix & (1u << j)) { R.a[j] = C.a[j]; R.b[j] = C.b[j]; }
    }
}

template <int NTX, int VY, bool EXACT, bool PRE = true>
__device__ __forceinline__ void st7_level(const Blk<double, VY>& ZM, const Blk<double, VY>& C,
                                          const Blk<double, VY>& ZP, const XN<double, VY>& xn, const Row<double>& top,
                                          const Row<double>& bot, const Coef<double>& k, bool yslow,
                                          uint32_t rowfix, Blk<double, VY>& R) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        const double left = PRE ? xn.l[j] : __shfl_up_sync(0xffffffffu, C.v[j][1], 1, NTX);
        const double right = PRE ? xn.r[j] : __shfl_down_sync(0xffffffffu, C.v[j][0], 1, NTX);
#pragma unroll
        for (int i = 0; i < 2; ++i) {
            const double c = C.v[j][i];
            const double xm = i == 0 ? left : C.v[j][0], xp = i == 1 ? right : C.v[j][1];
            const double ym = j > 0 ? C.v[j - 1][i] : top.v[i], yp = j < VY - 1 ? C.v[j + 1][i] : bot.v[i];
            const double sx = __dadd_rn(xm, xp), sy = __dadd_rn(ym, yp);
            if (!EXACT && ST_ZLAST) {   // z+1 term last (see the FP32 form)
                const double s = __dadd_rn(__dadd_rn(sy, sx), ZM.v[j][i]);
                R.v[j][i] = __fma_rn(k.be[i], ZP.v[j][i], __fma_rn(k.al[i], c, __dmul_rn(k.be[i], s)));
                continue;
            }
            const double sz = __dadd_rn(ZM.v[j][i], ZP.v[j][i]);
            const double s = __dadd_rn(__dadd_rn(sx, sy), sz);
            R.v[j][i] = EXACT ? __dadd_rn(__dmul_rn(k.al[i], c), __dmul_rn(k.be[i], s))
                              : __fma_rn(k.al[i], c, __dmul_rn(k.be[i], s));
        }
    }
    if (yslow) {
#pragma unroll
        for (int j = 0; j < VY; ++j)
            if (rowfix & (1u << j)) { R.v[j][0] = C.v[j][0]; R.v[j][1] = C.v[j][1]; }
    }
}

template <int NTX, int VY, bool EXACT, typename T>
__device__ __forceinline__ void st7_level(const Blk<T, VY>& ZM, const Blk<T, VY>& C, const Blk<T, VY>& ZP,
                                          const Row<T>& top, const Row<T>& bot, const Coef<T>& k, bool yslow,
                                          uint32_t rowfix, Blk<T, VY>& R) {
    st7_level<NTX, VY, EXACT, false>(ZM, C, ZP, XN<T, VY>{}, top, bot, k, yslow, rowfix, R);
}

template <typename T, int D, int NTX, int VY, bool EXACT, int MAXT>
__global__ void __launch_bounds__(MAXT, 1)
st7_35d_kernel(const __grid_constant__ CUtensorMap tmap, const St7Params p) {
    constexpr int VX = Vec<T>::N;
    constexpr int TX = NTX * VX;
    using V = typename Vec<T>::type;
    using B = Blk<T, VY>;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    const int tid = threadIdx.x;
    const int tx = tid % NTX;
    const int ty = tid / NTX;
    const int NTY = blockDim.x / NTX;
    const int TY = NTY * VY;
    const T al = T(p.alpha), be = T(p.beta);

    // the ring keeps the level-0 planes level 1 reads at round r: r-1 (its Y
    // neighbour rows) and r (ST7_L0REG: the Z window of level 0 is in registers),
    // or r-2, r-1, r (level 1 reads all three planes from shared memory)
    constexpr int KEEP = ST7_L0REG ? 2 : 3;
    const int RING = p.ring, PF = p.ring - KEEP;
    T* ring = reinterpret_cast<T*>(smem_raw);                      // [RING][TY][TX]
    const int slot_elems = TX * TY;
    // row exchange buffer [level 1..D-1][parity][N row / S row][MAXT] (16-byte rows)
    V* xbuf = reinterpret_cast<V*>(ring + RING * slot_elems);
    uint64_t* bars = reinterpret_cast<uint64_t*>(xbuf + (D > 1 ? (D - 1) * 4 * MAXT : 0));

    // zero the ring once: a boundary plane is formed as 1*c + 0*s and may read a
    // never-loaded neighbour plane slot, which must hold finite values
    for (int i = tid; i < RING * slot_elems * (int)sizeof(T) / 16; i += blockDim.x)
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

    // register planes: level l (1..D-1), rotating slot (prev / cur / new); level 0
    // is read straight from the TMA ring (index 0 unused)
    unsigned long long pr_t0 = ST7_PROF ? clock64() : 0, pr_wait = 0, pr_comp = 0, pr_bar = 0, pr_nr = 0, pr_ns = 0,
                       pr_ta = 0, pr_top = 0, pr_issue = 0, pr_gap = 0, pr_bend = 0;
    B pl[D][3];
    B outv;
#pragma unroll
    for (int l = 0; l < D; ++l)
#pragma unroll
        for (int k = 0; k < 3; ++k) pl[l][k] = B{};   // finite (see Coef)

    const int nzo = p.zb - p.za;
    long long item = p.split[blockIdx.x];
    const long long item_end = p.split[blockIdx.x + 1];
    const int zmin = max(0, -p.zbase);
    const int zmax = min(p.nzb - 1, p.nzg - 1 - p.zbase);
    const uint32_t tile_bytes = (uint32_t)(slot_elems * sizeof(T));
    uint32_t nload = 0;       // loads issued by this CTA so far (ring index)

    const int tyu = max(ty - 1, 0), tyd = min(ty + 1, NTY - 1);
    const int my_off = (VY * ty) * TX + VX * tx;                   // my first row in a plane
    const int top_off = max(VY * ty - 1, 0) * TX + VX * tx;         // row above my block
    const int bot_off = min(VY * ty + VY, TY - 1) * TX + VX * tx;   // row below my block
    V* const xw = xbuf + tid;                                      // my N row (S row at + MAXT)
    const V* const xtop = xbuf + MAXT + tyu * NTX + tx;            // S row of the block above
    const V* const xbot = xbuf + tyd * NTX + tx;                   // N row of the block below
    T* outp = reinterpret_cast<T*>(p.out);
    const size_t plane = (size_t)p.nx * p.ny;

    // segment = the part of this CTA's work range inside one tile: planes [za, zb)
    // of the output, level-0 planes [rl0, rl1] loaded at box corner (Lx, Ly)
    struct Seg { int tile, za, zb, Lx, Ly, rl0, rl1; };
    auto seg_at = [&](long long it) {
        Seg g;
        g.tile = (int)(it / nzo);
        const long long seg_end = min(item_end, (long long)(g.tile + 1) * nzo);
        g.za = p.za + (int)(it - (long long)g.tile * nzo);
        g.zb = p.za + (int)(seg_end - (long long)g.tile * nzo);
        g.Lx = (g.tile % p.tiles_x) * p.wx - p.hx;
        g.Ly = (g.tile / p.tiles_x) * p.wy - D;
        g.rl0 = max(g.za - D, zmin);
        g.rl1 = min(g.zb - 1 + D, zmax);
        return g;
    };
    int pre = 0;   // loads of the NEXT segment issued during this one's epilog (thread 0 only)

    unsigned long long pr_seg = 0, pr_first = 0;
    while (item < item_end) {
        const unsigned long long pr_ts = ST7_PROF ? clock64() : 0;
        const Seg sg = seg_at(item);
        const int tile = sg.tile, za = sg.za, zb = sg.zb;
        item += zb - za;
        // the next segment's first planes are loaded while this one drains
        const bool has_next = item < item_end;
        const Seg nx = seg_at(has_next ? item : item - 1);

        const int ix = tile % p.tiles_x, iy = tile / p.tiles_x;
        const int ox0 = ix * p.wx, ox1 = min(ox0 + p.wx, p.nx);
        const int oy0 = iy * p.wy, oy1 = min(oy0 + p.wy, p.ny);
        const int Lx = sg.Lx;
        const int Ly = sg.Ly;
        const int xg0 = Lx + VX * tx;
        uint32_t xfix = 0, rowfix = 0, rowmask = 0;
#pragma unroll
        for (int i = 0; i < VX; ++i)
            if (xg0 + i == 0 || xg0 + i == p.nx - 1) xfix |= 1u << i;
#pragma unroll
        for (int j = 0; j < VY; ++j) {
            const int yg = Ly + VY * ty + j;
            if (yg >= oy0 && yg < oy1) rowmask |= 1u << j;
            if (yg == 0 || yg == p.ny - 1) rowfix |= 1u << j;
        }
        const bool yslow = __any_sync(0xffffffffu, rowfix != 0);
        if (!(xg0 >= ox0 && xg0 < ox1)) rowmask = 0;    // quads are all-in or all-out in x
        const Coef<T> kc = Coef<T>::make(al, be, xfix);
        T* const outcol = outp + xg0 + (size_t)(Ly + VY * ty) * p.nx;

        // level-0 planes to load, rounds, and the steady rounds (every level
        // active, no z-shell plane): those run without any per-level check
        const int rl0 = sg.rl0;
        const int rl1 = sg.rl1;
        const int r0 = rl0;
        const int r1 = zb - 1 + D;
        const int rs0 = max(max(za + D, zmin + D), -p.zbase + D + 1);
        const int rs1 = min(min(zb - 1 + D, zmax + 1), min(rl1, p.nzg - 1 - p.zbase));
        const uint32_t kbase = nload;
        if (tid == 0) {
            for (int q = rl0 + pre; q <= min(rl0 + PF - 1, rl1); ++q) {
                const uint32_t k = kbase + (q - rl0);
                uint64_t* bar = &bars[k % RING];
                mbar_arrive_expect_tx(bar, tile_bytes);
                tma_load_3d(ring + (k % RING) * slot_elems, &tmap, bar, Lx, Ly, q);
            }
            pre = 0;
        }
        nload = kbase + (uint32_t)max(0, rl1 - rl0 + 1);
        // ring slot / parity of plane q, tracked incrementally (no division in the loop)
        uint32_t slot_r = kbase % RING, par_r = (kbase / RING) & 1;       // for plane r
        uint32_t slot_f = (kbase + PF) % RING;                            // for plane r + PF
        uint32_t slot_m1 = (slot_r + RING - 1) % RING;                    // for plane r - 1
        uint32_t slot_m2 = (slot_r + RING - 2) % RING;                    // for plane r - 2
        // output row pointer of plane r - D (level D at round r), advanced by one plane per round
        T* pout = outcol + (long long)(r0 - D) * (long long)plane;
        const int nxs = p.nx;

        auto round = [&](auto PHc, auto STEADYc, int r) {
            constexpr int PH = decltype(PHc)::value;
            constexpr bool STEADY = decltype(STEADYc)::value;
            // (a copy of the round loop without the per-level y-shell branch for
            // warps with no shell row was measured 25% SLOWER: the branch keeps
            // ptxas from interleaving levels, which costs registers and moves)
            const bool ysl = yslow;
            constexpr int PREV = PH % 3, CUR = (PH + 1) % 3, NEW = (PH + 2) % 3;
            if (ST7_PROF) { pr_top = clock64(); if (pr_bend) pr_gap += pr_top - pr_bend; }
            // issue the load of plane r + PF (its slot was freed by the barrier that ended round r-1)
            if (tid == 0) {
                if (r + PF <= rl1) {
                    uint64_t* bar = &bars[slot_f];
                    mbar_arrive_expect_tx(bar, tile_bytes);
                    tma_load_3d(ring + slot_f * slot_elems, &tmap, bar, Lx, Ly, r + PF);
                } else if (has_next && pre < PF && pre == r + PF - rl1 - 1 && nx.rl0 + pre <= nx.rl1) {
                    // slot_f holds ring sequence number kbase + (r + PF - rl0), which is the
                    // next segment's plane rl0' + pre (pre = r + PF - rl1 - 1): free since round r-1
                    uint64_t* bar = &bars[slot_f];
                    mbar_arrive_expect_tx(bar, tile_bytes);
                    tma_load_3d(ring + slot_f * slot_elems, &tmap, bar, nx.Lx, nx.Ly, nx.rl0 + pre);
                    ++pre;
                }
            }
            // level 0: plane r has landed in the ring
            if (ST7_PROF) { pr_ta = clock64(); pr_issue += pr_ta - pr_top; }
            if (STEADY || r <= rl1) mbar_wait(&bars[slot_r], par_r);
            unsigned long long pr_tb = 0;
            if (ST7_PROF) { pr_tb = clock64(); pr_wait += pr_tb - pr_ta; ++pr_nr; pr_ns += STEADY; }
            const int rpar = r & 1;
            if (ST7_L0REG && (STEADY || r <= rl1)) {   // level 0, plane r: my rows into the register Z window
                const T* s0 = ring + slot_r * slot_elems + my_off;
    #pragma unroll
                for (int j = 0; j < VY; ++j) pl[0][NEW].load_nat(j, s0 + j * TX);
            }
            // (The look-ahead exchange is measured faster for FP64 and VY = 2; the
            // FP32 VY = 4 blocks have no registers to spare and exchange per level.)
            if constexpr (sizeof(T) == 8 || VY == 2 || ST7_LOOKAHEAD) {
                // levels 1..D: level l computes plane z = r - l.  The X-neighbour
                // shuffles and exchange-row loads of level l+1 (whose centre plane
                // pl[l][CUR] exists since round r-1) are issued before level l computes.
                XN<T, VY> xnn;
                Row<T> tnn, bnn;
    #pragma unroll
                for (int l = 1; l <= D; ++l) {
                    if (ST7_DBG && (p.dbg & 1)) break;   // tuning build only: stream the planes without computing
                    const int z = r - l;
                    const int zpar = rpar ^ (l & 1);
                    const XN<T, VY> xnl = xnn;
                    const Row<T> tl = tnn, bl = bnn;
                    if (l < D) {
                        xnn = xshuf<NTX, VY>(pl[l][CUR]);
                        const int o = ((l - 1) * 4 + (zpar ^ 1) * 2) * MAXT;
                        tnn = row_x(xtop + o);
                        bnn = row_x(xbot + o);
                    }
                    bool zfix = false;
                    if (!STEADY) {
                        const int lo = max(za - (D - l), zmin), hi = min(zb - 1 + (D - l), zmax);
                        if (z < lo || z > hi) continue;
                        const int zg = p.zbase + z;
                        zfix = (zg == 0) || (zg == p.nzg - 1);
                    }
                    B& dst = l < D ? pl[l < D ? l : 1][NEW] : outv;
                    if (l == 1) {   // level-0 planes r-2, r-1, r of my block
                        const T* sl = ring + slot_m1 * slot_elems;   // level-0 neighbour rows of plane r-1
                        const Row<T> top = row_nat(sl + top_off), bot = row_nat(sl + bot_off);
                        B zm, c, zp;
                        if (ST7_L0REG) {
                            zm = pl[0][PREV]; c = pl[0][CUR]; zp = pl[0][NEW];
                        } else {
                            const T* s2 = ring + slot_m2 * slot_elems + my_off;
                            const T* s1 = ring + slot_m1 * slot_elems + my_off;
                            const T* s0 = ring + slot_r * slot_elems + my_off;
    #pragma unroll
                            for (int j = 0; j < VY; ++j) {
                                zm.load_nat(j, s2 + j * TX);
                                c.load_nat(j, s1 + j * TX);
                                zp.load_nat(j, s0 + j * TX);
                            }
                        }
                        const XN<T, VY> xc = xshuf<NTX, VY>(c);
                        if (!STEADY && zfix)
                            st7_level<NTX, VY, EXACT>(zm, c, zp, xc, top, bot, Coef<T>::fixed(), ysl, rowfix, dst);
                        else
                            st7_level<NTX, VY, EXACT>(zm, c, zp, xc, top, bot, kc, ysl, rowfix, dst);
                    } else {
                        const int lp = l > 1 ? l - 1 : 1;
                        if (!STEADY && zfix)
                            st7_level<NTX, VY, EXACT>(pl[lp][PREV], pl[lp][CUR], pl[lp][NEW], xnl, tl, bl,
                                                      Coef<T>::fixed(), ysl, rowfix, dst);
                        else
                            st7_level<NTX, VY, EXACT>(pl[lp][PREV], pl[lp][CUR], pl[lp][NEW], xnl, tl, bl, kc,
                                                      ysl, rowfix, dst);
                    }
                    if (l < D) {
                        V* xb = xw + ((l - 1) * 4 + zpar * 2) * MAXT;
                        dst.store_x(0, xb);
                        dst.store_x(VY - 1, xb + MAXT);
                    } else {
    #pragma unroll
                        for (int j = 0; j < VY; ++j)
                            if (rowmask & (1u << j)) outv.store_global(j, pout + j * nxs);
                    }
                }
            } else {
                // levels 1..D: level l computes plane z = r - l
    #pragma unroll
                for (int l = 1; l <= D; ++l) {
                    if (ST7_DBG && (p.dbg & 1)) break;   // tuning build only: stream the planes without computing
                    const int z = r - l;
                    bool zfix = false;
                    if (!STEADY) {
                        const int lo = max(za - (D - l), zmin), hi = min(zb - 1 + (D - l), zmax);
                        if (z < lo || z > hi) continue;
                        const int zg = p.zbase + z;
                        zfix = (zg == 0) || (zg == p.nzg - 1);
                    }
                    const int zpar = rpar ^ (l & 1);
                    Row<T> top, bot;
                    if (l == 1) {   // level-0 neighbours of plane r-1 straight from the TMA ring
                        const T* sl = ring + slot_m1 * slot_elems;
                        top = row_nat(sl + top_off);
                        bot = row_nat(sl + bot_off);
                    } else {        // rows exchanged by the blocks above / below in round r-1
                        const int o = ((l - 2) * 4 + zpar * 2) * MAXT;
                        top = row_x(xtop + o);
                        bot = row_x(xbot + o);
                    }
                    B& dst = l < D ? pl[l < D ? l : 1][NEW] : outv;
                    if (l == 1) {   // level-0 planes r-2, r-1, r of my block
                        B zm, c, zp;
                        if (ST7_L0REG) {
                            zm = pl[0][PREV]; c = pl[0][CUR]; zp = pl[0][NEW];
                        } else {
                            const T* s2 = ring + slot_m2 * slot_elems + my_off;
                            const T* s1 = ring + slot_m1 * slot_elems + my_off;
                            const T* s0 = ring + slot_r * slot_elems + my_off;
    #pragma unroll
                            for (int j = 0; j < VY; ++j) {
                                zm.load_nat(j, s2 + j * TX);
                                c.load_nat(j, s1 + j * TX);
                                zp.load_nat(j, s0 + j * TX);
                            }
                        }
                        if (!STEADY && zfix)
                            st7_level<NTX, VY, EXACT>(zm, c, zp, top, bot, Coef<T>::fixed(), ysl, rowfix, dst);
                        else
                            st7_level<NTX, VY, EXACT>(zm, c, zp, top, bot, kc, ysl, rowfix, dst);
                    } else {
                        const int lp = l > 1 ? l - 1 : 1;
                        if (!STEADY && zfix)
                            st7_level<NTX, VY, EXACT>(pl[lp][PREV], pl[lp][CUR], pl[lp][NEW], top, bot,
                                                      Coef<T>::fixed(), ysl, rowfix, dst);
                        else
                            st7_level<NTX, VY, EXACT>(pl[lp][PREV], pl[lp][CUR], pl[lp][NEW], top, bot, kc,
                                                      ysl, rowfix, dst);
                    }
                    if (l < D) {
                        V* xb = xw + ((l - 1) * 4 + zpar * 2) * MAXT;
                        dst.store_x(0, xb);
                        dst.store_x(VY - 1, xb + MAXT);
                    } else {
    #pragma unroll
                        for (int j = 0; j < VY; ++j)
                            if (rowmask & (1u << j)) outv.store_global(j, pout + j * nxs);
                    }
                }
            }
            unsigned long long pr_tc = 0;
            if (ST7_PROF) { pr_tc = clock64(); pr_comp += pr_tc - pr_tb; }
            __syncthreads();
            if (ST7_PROF) { pr_bend = clock64(); pr_bar += pr_bend - pr_tc; }
            pout += plane;
            // advance the ring cursors
            slot_m2 = slot_m1;
            slot_m1 = slot_r;
            if (++slot_r == (uint32_t)RING) { slot_r = 0; par_r ^= 1; }
            if (++slot_f == (uint32_t)RING) slot_f = 0;
        };
        using I0 = std::integral_constant<int, 0>;
        using I1 = std::integral_constant<int, 1>;
        using I2 = std::integral_constant<int, 2>;
        if (ST7_PROF) { const unsigned long long t = clock64(); pr_seg += t - pr_ts; if (!pr_first) pr_first = t - pr_t0; }
        if constexpr (ST7_STEADY_LOOP) {
        // Rounds of the steady range run as back-to-back phase triples with one
        // loop branch per three rounds; the other rounds (prolog, epilog, a
        // z-shell plane, and the few steady rounds before the phase wraps to 0)
        // take the checked path.  ph = (r - r0) mod 3 selects the register slots.
        int r = r0, ph = 0;
        while (r <= r1) {
            if (ph == 0 && r >= rs0 && r + 2 <= rs1) {
                do {
                    round(I0{}, std::true_type{}, r);
                    round(I1{}, std::true_type{}, r + 1);
                    round(I2{}, std::true_type{}, r + 2);
                    r += 3;
                } while (r + 2 <= rs1);
                continue;
            }
            const bool st = r >= rs0 && r <= rs1;
            if (ph == 0) { if (st) round(I0{}, std::true_type{}, r); else round(I0{}, std::false_type{}, r); }
            else if (ph == 1) { if (st) round(I1{}, std::true_type{}, r); else round(I1{}, std::false_type{}, r); }
            else { if (st) round(I2{}, std::true_type{}, r); else round(I2{}, std::false_type{}, r); }
            ++r;
            ph = ph == 2 ? 0 : ph + 1;
        }
        } else {
        auto any_round = [&](auto PHc, int r) {
            if (r >= rs0 && r <= rs1) round(PHc, std::true_type{}, r);
            else round(PHc, std::false_type{}, r);
        };
        for (int r = r0; r <= r1;) {
            any_round(I0{}, r);
            if (++r > r1) break;
            any_round(I1{}, r);
            if (++r > r1) break;
            any_round(I2{}, r);
            ++r;
        }
        }
    }
    if (ST7_PROF && p.prof && (tid & 31) == 0) {
        unsigned long long* o = p.prof + ((size_t)blockIdx.x * (MAXT / 32) + tid / 32) * 10;
        o[0] = clock64() - pr_t0; o[1] = pr_wait; o[2] = pr_comp; o[3] = pr_bar; o[4] = pr_nr; o[5] = pr_ns;
        o[6] = pr_seg; o[7] = pr_first; o[8] = pr_issue; o[9] = pr_gap;
    }
}

}  // namespace st35d
