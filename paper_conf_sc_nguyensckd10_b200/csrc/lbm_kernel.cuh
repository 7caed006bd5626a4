// lbm_kernel.cuh — D3Q19 lattice-Boltzmann step kernels for sm_100a.
//
// One step: read the 19 values and the flag of a cell,
// collide (BGK, X9), propagate the 19 new values to the 18
// neighbours and the cell itself; links into WALL cells bounce back, links
// into LID cells bounce back with the Ladd correction; non-FLUID cells keep
// their values.  The stored state is post-stream / pre-collision (X13).
//
// lbm_push_kernel (dim_T = 1 sweep): one thread per cell, SoA coalesced
// loads of the 19 populations, collision in registers,
// propagation as coalesced (x-shifted) stores — GPU stores do not
// write-allocate, so the paper's 228 B/update is 153 B here (X12).
//
// The collision arithmetic follows the oracle's operation order (X20); in
// bit-exact mode every operation is an explicitly rounded intrinsic, in the
// default mode the compiler may contract products into FMAs.
#pragma once
#include "common.cuh"


namespace st35d {

struct LbmParams {
    int nx, ny;
    int nzb;          // planes in the local buffers
    int zbase, nzg;   // global z of local plane 0, global nz
    int za, zb;       // local planes updated [za, zb)
    double omega;
    double lidc[19];  // (6 w_i)(e_i . u_lid), computed on the host in the plan dtype
};

// velocity set (X10): 0; +x -x +y -y +z -z; edges 7..18
__constant__ int8_t c_ex[19] = {0, 1, -1, 0, 0, 0, 0, 1, -1, 1, -1, 1, -1, 1, -1, 0, 0, 0, 0};
__constant__ int8_t c_ey[19] = {0, 0, 0, 1, -1, 0, 0, 1, -1, -1, 1, 0, 0, 0, 0, 1, -1, 1, -1};
__constant__ int8_t c_ez[19] = {0, 0, 0, 0, 0, 1, -1, 0, 0, 0, 0, 1, -1, -1, 1, 1, -1, -1, 1};

template <int I> struct D3Q19 {
    static constexpr int ex = (I == 1 || I == 7 || I == 9 || I == 11 || I == 13) ? 1
                            : (I == 2 || I == 8 || I == 10 || I == 12 || I == 14) ? -1 : 0;
    static constexpr int ey = (I == 3 || I == 7 || I == 10 || I == 15 || I == 17) ? 1
                            : (I == 4 || I == 8 || I == 9 || I == 16 || I == 18) ? -1 : 0;
    static constexpr int ez = (I == 5 || I == 11 || I == 14 || I == 15 || I == 18) ? 1
                            : (I == 6 || I == 12 || I == 13 || I == 16 || I == 17) ? -1 : 0;
    static constexpr int wden = I == 0 ? 3 : (I <= 6 ? 18 : 36);
    static constexpr int opp = I == 0 ? 0 : ((I & 1) ? I + 1 : I - 1);
};

template <typename T, bool EXACT> struct Ar;
template <bool E> struct Ar<float, E> {
    static __device__ __forceinline__ float add(float a, float b) { return E ? __fadd_rn(a, b) : a + b; }
    static __device__ __forceinline__ float sub(float a, float b) { return E ? __fsub_rn(a, b) : a - b; }
    static __device__ __forceinline__ float mul(float a, float b) { return E ? __fmul_rn(a, b) : a * b; }
    static __device__ __forceinline__ float div(float a, float b) { return __fdiv_rn(a, b); }
};
template <bool E> struct Ar<double, E> {
    static __device__ __forceinline__ double add(double a, double b) { return E ? __dadd_rn(a, b) : a + b; }
    static __device__ __forceinline__ double sub(double a, double b) { return E ? __dsub_rn(a, b) : a - b; }
    static __device__ __forceinline__ double mul(double a, double b) { return E ? __dmul_rn(a, b) : a * b; }
    static __device__ __forceinline__ double div(double a, double b) { return __ddiv_rn(a, b); }
};

template <typename T> struct Rcp;
template <> struct Rcp<float> { static __device__ __forceinline__ float rn(float x) { return __frcp_rn(x); } };
template <> struct Rcp<double> { static __device__ __forceinline__ double rn(double x) { return __drcp_rn(x); } };

// signed accumulation of e_a * f over the non-zero components, oracle order (X20)
template <typename T, bool E, int A, int I = 0>
__device__ __forceinline__ void jsum(const T (&f)[19], T& acc, bool& first) {
    if constexpr (I < 19) {
        constexpr int e = A == 0 ? D3Q19<I>::ex : (A == 1 ? D3Q19<I>::ey : D3Q19<I>::ez);
        if constexpr (e != 0) {
            if (first) { acc = e > 0 ? f[I] : -f[I]; first = false; }
            else acc = e > 0 ? Ar<T, E>::add(acc, f[I]) : Ar<T, E>::sub(acc, f[I]);
        }
        jsum<T, E, A, I + 1>(f, acc, first);
    }
}

template <typename T, bool E, int I>
__device__ __forceinline__ T edotu(T ux, T uy, T uz) {
    constexpr int ex = D3Q19<I>::ex, ey = D3Q19<I>::ey, ez = D3Q19<I>::ez;
    T eu = T(0);
    bool first = true;
    if constexpr (ex != 0) { eu = ex > 0 ? ux : -ux; first = false; }
    if constexpr (ey != 0) { T v = ey > 0 ? uy : -uy; eu = first ? v : Ar<T, E>::add(eu, v); first = false; }
    if constexpr (ez != 0) { T v = ez > 0 ? uz : -uz; eu = first ? v : Ar<T, E>::add(eu, v); first = false; }
    (void)first;
    return eu;
}

// BGK collision of one cell in place: f <- f - omega (f - feq), oracle order.
template <typename T, bool E>
__device__ __forceinline__ void collide(T (&f)[19], T omega) {
    using A = Ar<T, E>;
    T rho, jx, jy, jz;
    if (E) {   // oracle order (X20): sequential sums in index order
        rho = f[0];
#pragma unroll
        for (int i = 1; i < 19; ++i) rho = A::add(rho, f[i]);
        bool fx = true, fy = true, fz = true;
        jsum<T, E, 0>(f, jx, fx);
        jsum<T, E, 1>(f, jy, fy);
        jsum<T, E, 2>(f, jz, fz);
    } else {   // tolerance mode (X20): tree-ordered sums, depth 5 instead of 18
        const T s01 = f[1] + f[2], s34 = f[3] + f[4], s56 = f[5] + f[6];
        const T s78 = f[7] + f[8], s910 = f[9] + f[10], s1112 = f[11] + f[12], s1314 = f[13] + f[14];
        const T s1516 = f[15] + f[16], s1718 = f[17] + f[18];
        rho = ((f[0] + (s01 + s34)) + (s56 + s78)) + ((s910 + s1112) + (s1314 + (s1516 + s1718)));
        jx = ((f[1] - f[2]) + (f[7] - f[8])) + ((f[9] - f[10]) + ((f[11] - f[12]) + (f[13] - f[14])));
        jy = ((f[3] - f[4]) + (f[7] - f[8])) + ((f[10] - f[9]) + ((f[15] - f[16]) + (f[17] - f[18])));
        jz = ((f[5] - f[6]) + (f[11] - f[12])) + ((f[14] - f[13]) + ((f[15] - f[16]) + (f[18] - f[17])));
    }
    T ux, uy, uz;
    if (E) {   // oracle: three IEEE divisions
        ux = A::div(jx, rho); uy = A::div(jy, rho); uz = A::div(jz, rho);
    } else {   // tolerance mode: one correctly rounded reciprocal, three products
        const T inv = Rcp<T>::rn(rho);
        ux = jx * inv; uy = jy * inv; uz = jz * inv;
    }
    T usq = A::add(A::mul(ux, ux), A::mul(uy, uy));
    usq = A::add(usq, A::mul(uz, uz));
    const T usq15 = A::mul(T(1.5), usq);
    auto one = [&](auto Ic) {
        constexpr int I = decltype(Ic)::value;
        const T eu = edotu<T, E, I>(ux, uy, uz);
        const T w = T(1) / T(D3Q19<I>::wden);
        const T wr = A::mul(w, rho);
        const T a = A::add(T(1), A::mul(T(3), eu));
        const T c = A::mul(A::mul(T(4.5), eu), eu);
        const T g = A::sub(A::add(a, c), usq15);
        const T feq = A::mul(wr, g);
        f[I] = A::sub(f[I], A::mul(omega, A::sub(f[I], feq)));
    };
    [&]<int... Is>(std::integer_sequence<int, Is...>) { (one(std::integral_constant<int, Is>{}), ...); }
    (std::make_integer_sequence<int, 19>{});
}

// dim_T = 1: push form, one thread per cell, grid-stride over the updated planes.
// fl2 = flags | 0x80 for FLUID cells with a non-FLUID neighbour (lbm_fl2 prepass).
// Every store is predicated on the target cell's flag (WALL / LID links bounce
// back).  Measured on B200 (256^3 cavity, tools/lbm_ab.sh): an unconditional
// store path for interior cells is 20-35% SLOWER than flag-gated stores for
// FP32 — the gating paces the 19 stores of a cell behind short L1 hits instead
// of bursting them into the LSU queue ahead of other warps' loads — while
// FP64 (twice the bytes per store) prefers all 18 neighbour flags loaded up
// front (one round trip), 17.0 vs 15.7 GLUPS.
// constants of one push sweep (see lbm_push_kernel)
template <typename IX> struct PushCtx {
    size_t plane, lo0, lo1, hi0, hi1, last;
    IX ncx, pl;
    int nx;
};

// collide one cell (populations f, flag fl) and push its 19 values (or copy a
// non-FLUID cell through).  SLAB: only stores into the output planes are kept.
template <typename T, bool E, typename IX, bool BATCH, bool SLAB>
__device__ __forceinline__ void lbm_push_cell(T (&f)[19], uint32_t fl, size_t c, const uint8_t* __restrict__ fl2,
                                              T* __restrict__ dst, const PushCtx<IX>& k, T omega, const LbmParams& p) {
    const bool own = !SLAB || (c >= k.lo0 && c < k.hi1);
    const bool dn_ok = !SLAB || c >= k.lo1;     // target plane q-1 >= za
    const bool up_ok = !SLAB || c < k.hi0;      // target plane q+1 < zb
    T* __restrict__ d = dst + c;
    if (fl & 0x7fu) {   // WALL / LID: copied through
        if (own) {
#pragma unroll
            for (int i = 0; i < 19; ++i) d[(IX)i * k.ncx] = f[i];
        }
        return;
    }
    collide<T, E>(f, omega);
    uint32_t tfl[19];
    if constexpr (BATCH) {
        auto ld = [&](auto Ic) {
            constexpr int I = decltype(Ic)::value;
            const IX off = (IX)D3Q19<I>::ex + (IX)D3Q19<I>::ey * (IX)k.nx + (IX)D3Q19<I>::ez * k.pl;
            // (SLAB: a neighbour outside the buffer is never a store target; read nothing)
            const bool in = !SLAB || (D3Q19<I>::ez < 0 ? c >= k.plane : (D3Q19<I>::ez > 0 ? c < k.last : true));
            tfl[I] = (I == 0 || !in) ? 0u : (uint32_t)__ldg(fl2 + c + off);
        };
        [&]<int... Is>(std::integer_sequence<int, Is...>) { (ld(std::integral_constant<int, Is>{}), ...); }
        (std::make_integer_sequence<int, 19>{});
    }
    auto push = [&](auto Ic) {
        constexpr int I = decltype(Ic)::value;
        constexpr int ez = D3Q19<I>::ez;
        const IX off = (IX)D3Q19<I>::ex + (IX)D3Q19<I>::ey * (IX)k.nx + (IX)ez * k.pl;
        const bool tgt_ok = ez < 0 ? dn_ok : (ez > 0 ? up_ok : own);
        if constexpr (I == 0) {
            if (own) d[0] = f[0];
        } else {
            const bool in = !SLAB || (ez < 0 ? c >= k.plane : (ez > 0 ? c < k.last : true));
            const uint32_t tf = in ? (BATCH ? tfl[I] : (uint32_t)fl2[c + off]) & 0x7fu : 0u;
            if (tf == 0) { if (tgt_ok) d[(IX)I * k.ncx + off] = f[I]; }
            else if (!own) {}
            else if (tf == 1) d[(IX)D3Q19<I>::opp * k.ncx] = f[I];
            else d[(IX)D3Q19<I>::opp * k.ncx] = Ar<T, E>::sub(f[I], T(p.lidc[I]));
        }
    };
    [&]<int... Is>(std::integer_sequence<int, Is...>) { (push(std::integral_constant<int, Is>{}), ...); }
    (std::make_integer_sequence<int, 19>{});
}

template <typename IX>
__device__ __forceinline__ PushCtx<IX> push_ctx(const LbmParams& p, bool slab, int& pa, int& pb) {
    PushCtx<IX> k;
    k.plane = (size_t)p.nx * p.ny;
    const size_t nc = k.plane * p.nzb;               // SoA stride of one population
    pa = slab ? max(p.za - 1, 0) : p.za;
    pb = slab ? min(p.zb + 1, p.nzb) : p.zb;
    k.lo0 = (size_t)p.za * k.plane; k.lo1 = k.lo0 + k.plane;   // [lo0, lo1): plane za
    k.hi1 = (size_t)p.zb * k.plane; k.hi0 = k.hi1 - k.plane;   // [hi0, hi1): plane zb-1
    k.last = (size_t)(p.nzb - 1) * k.plane;
    k.ncx = (IX)nc; k.pl = (IX)k.plane;
    k.nx = p.nx;
    return k;
}

// SLAB (Z-slab sweeps): output planes [za, zb) of a buffer with
// ghost planes.  In push form a plane receives populations from its z
// neighbours, so source planes [za-1, zb+1) are processed and only stores whose
// target plane lies in [za, zb) are kept (each (cell, population) of the output
// planes is still written exactly once).  Single-domain sweeps have no ghosts:
// source and target ranges coincide and no store is filtered.
// CTAs per SM: per-direction flags 4 (64 registers); batched flags 3 for FP32
// (80 registers) and 2 for FP64 (128 registers), all without spills
template <typename T> constexpr int lbm_push_ctas(bool batch) { return batch ? (sizeof(T) == 4 ? 3 : 2) : 4; }

template <typename T, bool E, typename IX, bool BATCH, bool SLAB>
__global__ void __launch_bounds__(256, lbm_push_ctas<T>(BATCH))
lbm_push_kernel(const T* __restrict__ src, T* __restrict__ dst, const uint8_t* __restrict__ fl2,
                const LbmParams p) {
    int pa, pb;
    const PushCtx<IX> k = push_ctx<IX>(p, SLAB, pa, pb);
    const size_t c0 = (size_t)pa * k.plane;
    const size_t ncell = (size_t)(pb - pa) * k.plane;
    const T omega = T(p.omega);
    for (size_t t = blockIdx.x * (size_t)blockDim.x + threadIdx.x; t < ncell; t += (size_t)gridDim.x * blockDim.x) {
        const size_t c = c0 + t;
        const uint32_t fl = fl2[c];
        const T* __restrict__ s = src + c;
        T f[19];
#pragma unroll
        for (int i = 0; i < 19; ++i) f[i] = s[(IX)i * k.ncx];
        lbm_push_cell<T, E, IX, BATCH, SLAB>(f, fl, c, fl2, dst, k, omega, p);
    }
}


// ---------------------------------------------------------------------------
// Gather form (a10: every store of a cell's 19 values is aligned and
// coalesced at the cell itself, no x-shifted scatter).  With P = S.C the push
// step (collide, then stream), T push steps are  P^T = S . (C.S)^(T-1) . C:
// one collide-only pass, T-1 pull passes (gather the neighbours'
// post-collision values, then collide) and one stream-only pass.  The stored
// intermediate state is post-collision; every (cell, population) sees the
// same operations as in the push kernel, so the result is bit-identical.
// Bounce-back in gather form: the value arriving at x in direction i comes
// from x - e_i; if that cell is WALL it is x's own post-collision value of
// opp(i) (the half-way reflection), if LID the same minus (6 w e.u)_opp(i).
// fl2 marks FLUID cells with a non-FLUID neighbour; only they read flags.
// ---------------------------------------------------------------------------
enum { LBM_COLLIDE = 0, LBM_PULL = 1, LBM_STREAM = 2 };

template <typename T, bool E, int MODE>
__global__ void __launch_bounds__(256, 4)
lbm_gather_kernel(const T* src, T* dst, const uint8_t* __restrict__ fl2, const LbmParams p) {
    // (src may equal dst for the in-place collide pass: no __restrict__ on the lattices)
    const size_t plane = (size_t)p.nx * p.ny;
    const long long nc = (long long)(plane * p.nzb);
    const size_t c0 = (size_t)p.za * plane;
    const size_t ncell = (size_t)(p.zb - p.za) * plane;
    const T omega = T(p.omega);
    for (size_t t = blockIdx.x * (size_t)blockDim.x + threadIdx.x; t < ncell; t += (size_t)gridDim.x * blockDim.x) {
        const size_t c = c0 + t;
        const uint32_t fl = fl2[c];
        const T* s = src + c;
        T* d = dst + c;
        T f[19];
        if ((fl & 0x7fu) != 0 || MODE == LBM_COLLIDE) {
#pragma unroll
            for (int i = 0; i < 19; ++i) f[i] = s[(long long)i * nc];
            if ((fl & 0x7fu) == 0) collide<T, E>(f, omega);   // COLLIDE on a FLUID cell
#pragma unroll
            for (int i = 0; i < 19; ++i) d[(long long)i * nc] = f[i];
            continue;
        }
        auto gather = [&](auto Ic) {
            constexpr int I = decltype(Ic)::value;
            const long long off = (long long)D3Q19<I>::ex + (long long)D3Q19<I>::ey * p.nx +
                                  (long long)D3Q19<I>::ez * (long long)plane;
            if constexpr (I == 0) {
                f[0] = s[0];
            } else {
                const uint32_t sf = (fl & 0x80u) ? (uint32_t)__ldg(fl2 + (long long)c - off) & 0x7fu : 0u;
                if (sf == 0) f[I] = s[(long long)I * nc - off];
                else if (sf == 1) f[I] = s[(long long)D3Q19<I>::opp * nc];
                else f[I] = Ar<T, E>::sub(s[(long long)D3Q19<I>::opp * nc], T(p.lidc[D3Q19<I>::opp]));
            }
        };
        [&]<int... Is>(std::integer_sequence<int, Is...>) { (gather(std::integral_constant<int, Is>{}), ...); }
        (std::make_integer_sequence<int, 19>{});
        if (MODE == LBM_PULL) collide<T, E>(f, omega);
#pragma unroll
        for (int i = 0; i < 19; ++i) d[(long long)i * nc] = f[i];
    }
}

// ---------------------------------------------------------------------------
// lbm_35d_kernel: the 3.5D-blocked D3Q19 sweep (dim_T = D levels on chip).
//
// A CTA owns a 32 x TY cell tile (one cell per thread, a warp = one row) of
// an XY sub-plane and streams it along Z.  Transition l (level
// l-1 -> l) at round r takes the level-(l-1) plane q = r-l+1, collides every
// FLUID cell (BGK, X9) and PUSHES the 19 post-collision values
// into level l's planes q-1, q, q+1; a push into a WALL / LID cell bounces
// back into the cell's own opposite population (X10).  Level l's plane r-l is
// then complete (its three source planes were processed in rounds r-2..r),
// so lag 1 per level and one barrier per transition.  Levels 1..D-1 are
// assembled in a 3-plane shared-memory ring per level (padded by one cell so
// edge pushes stay in bounds); the last transition pushes straight into the
// output lattice, only for target cells in the tile's written region
// (X - 2D) x (Y - 2D) and the segment's planes, so every (cell, population)
// of f_dst is written exactly once.  Level 0 is read with coalesced SoA loads,
// prefetched one plane ahead into registers.
// fl2 = flags | 0x80 for a FLUID cell with a non-FLUID neighbour (host prepass):
// only those cells look at their neighbours' flags.
// ---------------------------------------------------------------------------
struct Lbm35Params {
    const void* src;
    void* dst;
    const uint8_t* fl2;
    int nx, ny, nzb, zbase, nzg, za, zb;
    int tiles_x, wx, wy;
    long long work;
    double omega;
    double lidc[19];
};

template <int I, typename T, bool E, typename F>
__device__ __forceinline__ void lbm_push_one(const T (&fs)[19], uint32_t fl, int x, int y, int q, int nx, int ny,
                                             int nzb, size_t plane, const uint8_t* __restrict__ fl2, const T* lidc,
                                             F&& put) {
    constexpr int ex = D3Q19<I>::ex, ey = D3Q19<I>::ey, ez = D3Q19<I>::ez;
    if constexpr (I == 0) {
        put(0, 0, 0, 0, fs[0]);
    } else {
        uint32_t tf = 0;   // a neighbour outside the slab buffer is a ghost-side cell: never non-FLUID here
        if ((fl & 0x80u) && q + ez >= 0 && q + ez < nzb)
            tf = __ldg(fl2 + (size_t)(q + ez) * plane + (size_t)(y + ey) * nx + (x + ex)) & 0x7fu;
        if (tf == 0) put(I, ex, ey, ez, fs[I]);
        else if (tf == 1) put(D3Q19<I>::opp, 0, 0, 0, fs[I]);
        else put(D3Q19<I>::opp, 0, 0, 0, Ar<T, E>::sub(fs[I], lidc[I]));
    }
}

template <typename T, int D, bool E>
__global__ void __launch_bounds__(512, 1) lbm_35d_kernel(const Lbm35Params p) {
    constexpr int TX = 32, PX = TX + 2;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    const int TY = blockDim.x >> 5, PY = TY + 2;
    const int pstride = PX * PY;                 // one population plane of the padded tile
    const int sstride = 19 * pstride;            // one ring slot
    T* asmb = reinterpret_cast<T*>(smem_raw);    // [D-1][3][19][PY][PX]
    const T* __restrict__ src = static_cast<const T*>(p.src);
    T* __restrict__ dst = static_cast<T*>(p.dst);
    const size_t plane = (size_t)p.nx * p.ny;
    const size_t nc = plane * p.nzb;
    const T omega = T(p.omega);
    T lidc[19];
#pragma unroll
    for (int i = 0; i < 19; ++i) lidc[i] = T(p.lidc[i]);
    const int zmin = max(0, -p.zbase);
    const int zmax = min(p.nzb - 1, p.nzg - 1 - p.zbase);
    const int nzo = p.zb - p.za;
    const long long G = gridDim.x;
    long long item = p.work * (long long)blockIdx.x / G;
    const long long item_end = p.work * ((long long)blockIdx.x + 1) / G;
    const int me = (ty + 1) * PX + (tx + 1);     // my cell in a padded population plane

    while (item < item_end) {
        const int tile = (int)(item / nzo);
        const long long seg_end = min(item_end, (long long)(tile + 1) * nzo);
        const int za = p.za + (int)(item - (long long)tile * nzo);
        const int zb = p.za + (int)(seg_end - (long long)tile * nzo);
        item = seg_end;
        const int ix = tile % p.tiles_x, iy = tile / p.tiles_x;
        const int ox0 = ix * p.wx, ox1 = min(ox0 + p.wx, p.nx);
        const int oy0 = iy * p.wy, oy1 = min(oy0 + p.wy, p.ny);
        const int x = ox0 - D + tx, y = oy0 - D + ty;
        const bool inb = x >= 0 && x < p.nx && y >= 0 && y < p.ny;
        const size_t cxy = inb ? (size_t)y * p.nx + x : 0;
        const int rl0 = max(za - D, zmin), rl1 = min(zb - 1 + D, zmax);

        T fnext[19];
        uint32_t flnext = 0;
        auto load = [&](int q) {
            if (inb && q <= rl1) {
                const size_t c = (size_t)q * plane + cxy;
#pragma unroll
                for (int i = 0; i < 19; ++i) fnext[i] = src[i * nc + c];
                flnext = p.fl2[c];
            }
        };
        load(rl0);
        uint64_t flh = 0;   // own flags of the last 8 level-0 planes (byte k = plane r-k)

        for (int r = rl0; r <= zb - 1 + D; ++r) {
            T f[19];
#pragma unroll
            for (int i = 0; i < 19; ++i) f[i] = fnext[i];
            flh = (flh << 8) | (r <= rl1 ? flnext : 0u);
            load(r + 1);
#pragma unroll
            for (int l = 1; l <= D; ++l) {
                const int q = r - l + 1;                                 // level-(l-1) plane processed
                const int lo = max(za - D + l - 1, zmin), hi = min(zb + D - l, zmax);
                if (q >= lo && q <= hi && inb) {
                    if (l > 1) {   // level l-1 plane q from the assembly ring
                        const T* a = asmb + ((size_t)(l - 2) * 3 + (size_t)(q % 3)) * sstride + me;
#pragma unroll
                        for (int i = 0; i < 19; ++i) f[i] = a[i * pstride];
                    }
                    const uint32_t fl = (uint32_t)(flh >> (8 * (l - 1))) & 0xffu;
                    if (l < D) {
                        T* ab = asmb + (size_t)(l - 1) * 3 * sstride;
                        auto put = [&](int pop, int ex, int ey, int ez, T v) {
                            ab[(size_t)((q + ez + 3) % 3) * sstride + pop * pstride + me + ey * PX + ex] = v;
                        };
                        if ((fl & 0x7fu) != 0) {
#pragma unroll
                            for (int i = 0; i < 19; ++i) put(i, 0, 0, 0, f[i]);
                        } else {
                            collide<T, E>(f, omega);
                            [&]<int... Is>(std::integer_sequence<int, Is...>) {
                                (lbm_push_one<Is, T, E>(f, fl, x, y, q, p.nx, p.ny, p.nzb, plane, p.fl2, lidc, put), ...);
                            }(std::make_integer_sequence<int, 19>{});
                        }
                    } else {
                        const size_t cq = (size_t)q * plane + cxy;
                        auto put = [&](int pop, int ex, int ey, int ez, T v) {
                            const int tx2 = x + ex, ty2 = y + ey, tz = q + ez;
                            if (tx2 >= ox0 && tx2 < ox1 && ty2 >= oy0 && ty2 < oy1 && tz >= za && tz < zb)
                                dst[pop * nc + (size_t)((long long)cq + ex + (long long)ey * p.nx +
                                                        (long long)ez * (long long)plane)] = v;
                        };
                        if ((fl & 0x7fu) != 0) {
#pragma unroll
                            for (int i = 0; i < 19; ++i) put(i, 0, 0, 0, f[i]);
                        } else {
                            collide<T, E>(f, omega);
                            [&]<int... Is>(std::integer_sequence<int, Is...>) {
                                (lbm_push_one<Is, T, E>(f, fl, x, y, q, p.nx, p.ny, p.nzb, plane, p.fl2, lidc, put), ...);
                            }(std::make_integer_sequence<int, 19>{});
                        }
                    }
                }
                if (D > 1) __syncthreads();
            }
        }
    }
}

}  // namespace st35d
