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

namespace st35d {

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
    double alpha, beta;
};

constexpr int ST7_RING = 4;   // TMA ring slots
constexpr int ST7_PF = 2;     // planes prefetched ahead

template <typename T>
__device__ __forceinline__ T st7_point(T c, T xm, T xp, T ym, T yp, T zm, T zp, T al, T be, bool exact) {
    if (exact) {
        // oracle order (X2): ((x- + x+) + (y- + y+)) + (z- + z+); two products, one add
        T sx = __dadd_rn(xm, xp), sy = __dadd_rn(ym, yp), sz = __dadd_rn(zm, zp);
        T s = __dadd_rn(__dadd_rn(sx, sy), sz);
        return __dadd_rn(__dmul_rn(al, c), __dmul_rn(be, s));
    } else {
        T s = ((xm + xp) + (ym + yp)) + (zm + zp);
        return fma(al, c, be * s);
    }
}
template <>
__device__ __forceinline__ float st7_point<float>(float c, float xm, float xp, float ym, float yp, float zm,
                                                  float zp, float al, float be, bool exact) {
    if (exact) {
        float sx = __fadd_rn(xm, xp), sy = __fadd_rn(ym, yp), sz = __fadd_rn(zm, zp);
        float s = __fadd_rn(__fadd_rn(sx, sy), sz);
        return __fadd_rn(__fmul_rn(al, c), __fmul_rn(be, s));
    } else {
        float s = ((xm + xp) + (ym + yp)) + (zm + zp);
        return fmaf(al, c, be * s);
    }
}

template <typename T, int VX>
__device__ __forceinline__ void vload(T (&dst)[VX], const T* src) {
    using V = typename Vec<T>::type;
    V v = *reinterpret_cast<const V*>(src);
    if constexpr (VX == 4) { dst[0] = v.x; dst[1] = v.y; dst[2] = v.z; dst[3] = v.w; }
    else { dst[0] = v.x; dst[1] = v.y; }
}
template <typename T, int VX>
__device__ __forceinline__ void vstore(T* dst, const T (&s)[VX]) {
    using V = typename Vec<T>::type;
    if constexpr (VX == 4) *reinterpret_cast<V*>(dst) = V{s[0], s[1], s[2], s[3]};
    else *reinterpret_cast<V*>(dst) = V{s[0], s[1]};
}
template <typename T, int VX>
__device__ __forceinline__ void gstore(T* dst, const T (&s)[VX]) {
    if constexpr (VX == 4) st_global_v4(reinterpret_cast<float*>(dst), make_float4(s[0], s[1], s[2], s[3]));
    else st_global_v2(reinterpret_cast<double*>(dst), make_double2(s[0], s[1]));
}

template <typename T, int D, int NTX, int VY, bool EXACT>
struct St7Sweep {
    static constexpr int VX = Vec<T>::N;
    static constexpr int TX = NTX * VX;

    // per-thread register planes: level l (0..D-1), rotating slot k (0..2)
    T pl[D][3][VY][VX];
    T outv[VY][VX];

    // block geometry
    int tx, ty, NTY, TY;
    // segment geometry
    int Lx, Ly, ox0, ox1, oy0, oy1;
    uint32_t fixmask;      // bit j*VX+i: point is on the grid shell or outside (copied)
    bool wfix;             // warp-uniform: some lane of the warp has fixmask != 0
    T al, be;

    __device__ __forceinline__ void compute_level(const T (&ZM)[VY][VX], const T (&C)[VY][VX],
                                                  const T (&ZP)[VY][VX], const T* top, const T* bot,
                                                  bool zfix, T (&R)[VY][VX]) {
        T up[VX], dn[VX];
#pragma unroll
        for (int i = 0; i < VX; ++i) { up[i] = top[i]; dn[i] = bot[i]; }
        T left[VY], right[VY];
#pragma unroll
        for (int j = 0; j < VY; ++j) {
            left[j] = __shfl_up_sync(0xffffffffu, C[j][VX - 1], 1, NTX);
            right[j] = __shfl_down_sync(0xffffffffu, C[j][0], 1, NTX);
        }
        if (zfix) {
#pragma unroll
            for (int j = 0; j < VY; ++j)
#pragma unroll
                for (int i = 0; i < VX; ++i) R[j][i] = C[j][i];
            return;
        }
#pragma unroll
        for (int j = 0; j < VY; ++j)
#pragma unroll
            for (int i = 0; i < VX; ++i) {
                T xm = i > 0 ? C[j][i - 1] : left[j];
                T xp = i < VX - 1 ? C[j][i + 1] : right[j];
                T ym = j > 0 ? C[j - 1][i] : up[i];
                T yp = j < VY - 1 ? C[j + 1][i] : dn[i];
                R[j][i] = st7_point<T>(C[j][i], xm, xp, ym, yp, ZM[j][i], ZP[j][i], al, be, EXACT);
            }
        if (wfix) {  // warp-uniform: only warps touching the grid shell pay for the selects
#pragma unroll
            for (int j = 0; j < VY; ++j)
#pragma unroll
                for (int i = 0; i < VX; ++i)
                    if (fixmask & (1u << (j * VX + i))) R[j][i] = C[j][i];
        }
    }
};

template <typename T, int D, int NTX, int VY, bool EXACT, int MAXT>
__global__ void __launch_bounds__(MAXT, 1)
st7_35d_kernel(const __grid_constant__ CUtensorMap tmap, const St7Params p) {
    using S = St7Sweep<T, D, NTX, VY, EXACT>;
    constexpr int VX = S::VX;
    constexpr int TX = S::TX;
    using V = typename Vec<T>::type;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    S st;
    st.tx = threadIdx.x % NTX;
    st.ty = threadIdx.x / NTX;
    st.NTY = blockDim.x / NTX;
    st.TY = st.NTY * VY;
    const int NT = blockDim.x;
    const int TY = st.TY;
    st.al = T(p.alpha);
    st.be = T(p.beta);

    T* ring = reinterpret_cast<T*>(smem_raw);                      // [ST7_RING][TY][TX]
    const int slot_elems = TX * TY;
    V* xbuf = reinterpret_cast<V*>(ring + ST7_RING * slot_elems);  // [D-1][2 parity][2 N/S][NT]
    uint64_t* bars = reinterpret_cast<uint64_t*>(xbuf + (D > 1 ? (D - 1) * 4 * NT : 0));

    if (threadIdx.x == 0) {
        prefetch_tensormap(&tmap);
        for (int s = 0; s < ST7_RING; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
    }
    __syncthreads();

    const int nzo = p.zb - p.za;
    const long long G = gridDim.x;
    long long item = p.work * (long long)blockIdx.x / G;
    const long long item_end = p.work * ((long long)blockIdx.x + 1) / G;
    const int zmin = max(0, -p.zbase);
    const int zmax = min(p.nzb - 1, p.nzg - 1 - p.zbase);
    const uint32_t tile_bytes = (uint32_t)(slot_elems * sizeof(T));
    uint32_t nload = 0;       // loads issued by this CTA so far (ring index)

    const int tyu = max(st.ty - 1, 0), tyd = min(st.ty + 1, st.NTY - 1);
    const int my_off = (VY * st.ty) * TX + VX * st.tx;                 // my first row in a plane
    const int top_off = max(VY * st.ty - 1, 0) * TX + VX * st.tx;       // row above my block
    const int bot_off = min(VY * st.ty + VY, TY - 1) * TX + VX * st.tx; // row below my block
    T* outp = reinterpret_cast<T*>(p.out);
    const size_t plane = (size_t)p.nx * p.ny;

    while (item < item_end) {
        const int tile = (int)(item / nzo);
        const long long tile_end = (long long)(tile + 1) * nzo;
        const long long seg_end = min(item_end, tile_end);
        const int za = p.za + (int)(item - (long long)tile * nzo);
        const int zb = p.za + (int)(seg_end - (long long)tile * nzo);
        item = seg_end;

        const int ix = tile % p.tiles_x, iy = tile / p.tiles_x;
        st.ox0 = ix * p.wx; st.ox1 = min(st.ox0 + p.wx, p.nx);
        st.oy0 = iy * p.wy; st.oy1 = min(st.oy0 + p.wy, p.ny);
        st.Lx = st.ox0 - p.hx;
        st.Ly = st.oy0 - D;
        st.fixmask = 0;
#pragma unroll
        for (int j = 0; j < VY; ++j)
#pragma unroll
            for (int i = 0; i < VX; ++i) {
                int xg = st.Lx + VX * st.tx + i, yg = st.Ly + VY * st.ty + j;
                bool interior = xg >= 1 && xg <= p.nx - 2 && yg >= 1 && yg <= p.ny - 2;
                if (!interior) st.fixmask |= 1u << (j * VX + i);
            }
        st.wfix = __any_sync(0xffffffffu, st.fixmask != 0);

        // level-0 planes to load, and rounds
        const int rl0 = max(za - D, zmin);
        const int rl1 = min(zb - 1 + D, zmax);
        const int r0 = rl0;
        const int r1 = zb - 1 + D;
        const uint32_t kbase = nload;
        if (threadIdx.x == 0) {
            for (int q = rl0; q <= min(rl0 + ST7_PF - 1, rl1); ++q) {
                uint32_t k = kbase + (q - rl0);
                uint64_t* bar = &bars[k % ST7_RING];
                mbar_arrive_expect_tx(bar, tile_bytes);
                tma_load_3d(ring + (k % ST7_RING) * slot_elems, &tmap, bar, st.Lx, st.Ly, q);
            }
        }
        nload = kbase + (uint32_t)max(0, rl1 - rl0 + 1);

        auto round = [&](auto PHc, int r) {
            constexpr int PH = decltype(PHc)::value;
            constexpr int PREV = PH % 3, CUR = (PH + 1) % 3, NEW = (PH + 2) % 3;
            // issue the load of plane r + PF (slot freed by the barrier that ended round r-1)
            if (threadIdx.x == 0 && r + ST7_PF <= rl1) {
                uint32_t k = kbase + (r + ST7_PF - rl0);
                uint64_t* bar = &bars[k % ST7_RING];
                mbar_arrive_expect_tx(bar, tile_bytes);
                tma_load_3d(ring + (k % ST7_RING) * slot_elems, &tmap, bar, st.Lx, st.Ly, r + ST7_PF);
            }
            // level 0: plane r from the ring into registers
            if (r <= rl1) {
                uint32_t k = kbase + (r - rl0);
                mbar_wait(&bars[k % ST7_RING], (k / ST7_RING) & 1);
                const T* sl = ring + (k % ST7_RING) * slot_elems;
#pragma unroll
                for (int j = 0; j < VY; ++j) vload<T, VX>(st.pl[0][NEW][j], sl + my_off + j * TX);
            }
            // levels 1..D: level l computes plane r - l
#pragma unroll
            for (int l = 1; l <= D; ++l) {
                const int z = r - l;
                const int lo = max(za - (D - l), zmin), hi = min(zb - 1 + (D - l), zmax);
                if (z < lo || z > hi) continue;
                const int zg = p.zbase + z;
                const bool zfix = (zg == 0) || (zg == p.nzg - 1);
                const T* top;
                const T* bot;
                if (l == 1) {
                    uint32_t k = kbase + (z - rl0);
                    const T* sl = ring + (k % ST7_RING) * slot_elems;
                    top = sl + top_off;
                    bot = sl + bot_off;
                } else {
                    const V* xb = xbuf + ((size_t)(l - 2) * 4 + (z & 1) * 2) * NT;
                    top = reinterpret_cast<const T*>(xb + NT + tyu * NTX + st.tx);   // S-row of block above
                    bot = reinterpret_cast<const T*>(xb + tyd * NTX + st.tx);        // N-row of block below
                }
                if (l < D) {
                    st.compute_level(st.pl[l - 1][PREV], st.pl[l - 1][CUR], st.pl[l - 1][NEW], top, bot, zfix,
                                     st.pl[l][NEW]);
                    V* xb = xbuf + ((size_t)(l - 1) * 4 + (z & 1) * 2) * NT;
                    vstore<T, VX>(reinterpret_cast<T*>(xb + threadIdx.x), st.pl[l][NEW][0]);
                    vstore<T, VX>(reinterpret_cast<T*>(xb + NT + threadIdx.x), st.pl[l][NEW][VY - 1]);
                } else {
                    st.compute_level(st.pl[l - 1][PREV], st.pl[l - 1][CUR], st.pl[l - 1][NEW], top, bot, zfix,
                                     st.outv);
                    const int xg = st.Lx + VX * st.tx;
                    if (xg >= st.ox0 && xg < st.ox1) {
                        T* base = outp + (size_t)z * plane + xg;
#pragma unroll
                        for (int j = 0; j < VY; ++j) {
                            const int yg = st.Ly + VY * st.ty + j;
                            if (yg >= st.oy0 && yg < st.oy1) gstore<T, VX>(base + (size_t)yg * p.nx, st.outv[j]);
                        }
                    }
                }
            }
            __syncthreads();
        };

        for (int r = r0; r <= r1;) {
            round(std::integral_constant<int, 0>{}, r);
            if (++r > r1) break;
            round(std::integral_constant<int, 1>{}, r);
            if (++r > r1) break;
            round(std::integral_constant<int, 2>{}, r);
            ++r;
        }
    }
}

}  // namespace st35d
