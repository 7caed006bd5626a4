// st13_kernel.cuh — 3.5D-blocked radius-2 (13-point star) Jacobi sweep for
// sm_100a: the general stencil radius R of §V with R = 2 (SURVEY §8(f)
// f4; readings X25 weights / order, X26 2-point-thick fixed shell).
//
// Same machinery as the 7-point kernel (st7_kernel.cuh: persistent CTAs over
// equal-cost (tile, z) work, a TMA plane ring with mbarriers, a register Z
// window, X neighbours by shuffle, Y neighbours through a row exchange,
// two-phase rounds), with the changes R = 2 brings (X5):
//  * lag R per level: level l at round r computes plane q = r - 2l; its
//    planes q-2 .. q+1 of level l-1 are in registers and q+2 is the plane
//    level l-1 produces in the same round (the paper's z_s = z + 2R(dim_T - t'),
//    P:251, runs the levels 2R apart because its buffers are shared caches;
//    with the window in registers R planes per level suffice);
//  * a 5-slot register window per level (2R+1 planes), rotated at compile
//    time by unrolling the steady rounds by 5;
//  * the halo is R*dim_T points per side; the Y exchange carries R rows per
//    side and waits two rounds (three exchange buffers, the in-plane
//    neighbours of plane q are produced in round r-2);
//  * the ring keeps planes r-2 .. r (level 1's centre plane is r-2).
// Update (fast): A = alpha*c + beta*((x1 + y1) + (zm1 + zp1)) + gamma*((x2 + y2) + zm2)
// in phase A, out = A + gamma*zp2 in phase C; exact: the oracle's
// p = alpha*c + beta*S1 in phase A, then (p + gamma*S2) with S2 completed by
// (z-2 + z+2) in phase C, every operation rounded (oracle_st13).
#pragma once
#include "st7_kernel.cuh"

namespace st35d {

constexpr int ST13_R = 2;

// one row's X neighbours at distance 1 and 2 from the adjacent lanes
template <int NTX, int VY>
__device__ __forceinline__ void xshfl2(const Bk<float, VY>& H, float2 (&L)[VY], float2 (&R)[VY]) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {   // L = (c2, c3) of the left lane, R = (c0, c1) of the right lane
        L[j] = make_float2(__shfl_up_sync(0xffffffffu, H.r[j].b.x, 1, NTX), __shfl_up_sync(0xffffffffu, H.r[j].b.y, 1, NTX));
        R[j] = make_float2(__shfl_down_sync(0xffffffffu, H.r[j].a.x, 1, NTX),
                           __shfl_down_sync(0xffffffffu, H.r[j].a.y, 1, NTX));
    }
}
template <int NTX, int VY>
__device__ __forceinline__ void xshfl2(const Bk<double, VY>& H, double2 (&L)[VY], double2 (&R)[VY]) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {   // L = (c0, c1) of the left lane, R = (c0, c1) of the right lane
        L[j] = make_double2(__shfl_up_sync(0xffffffffu, H.r[j].x0, 1, NTX), __shfl_up_sync(0xffffffffu, H.r[j].x1, 1, NTX));
        R[j] = make_double2(__shfl_down_sync(0xffffffffu, H.r[j].x0, 1, NTX),
                            __shfl_down_sync(0xffffffffu, H.r[j].x1, 1, NTX));
    }
}

// per-lane coefficients; an x-shell column (x < 2 or x >= nx-2) gets (1, 0, 0)
template <typename T> struct St13Coef;
template <> struct St13Coef<float> {
    float2 alA, beA, gaA, alB, beB, gaB;
    static __device__ __forceinline__ St13Coef make(float al, float be, float ga, uint32_t xfix) {
        St13Coef k;
        k.alA = make_float2(xfix & 1 ? 1.f : al, xfix & 2 ? 1.f : al);
        k.beA = make_float2(xfix & 1 ? 0.f : be, xfix & 2 ? 0.f : be);
        k.gaA = make_float2(xfix & 1 ? 0.f : ga, xfix & 2 ? 0.f : ga);
        k.alB = make_float2(xfix & 4 ? 1.f : al, xfix & 8 ? 1.f : al);
        k.beB = make_float2(xfix & 4 ? 0.f : be, xfix & 8 ? 0.f : be);
        k.gaB = make_float2(xfix & 4 ? 0.f : ga, xfix & 8 ? 0.f : ga);
        return k;
    }
};
template <> struct St13Coef<double> {
    double al0, be0, ga0, al1, be1, ga1;
    static __device__ __forceinline__ St13Coef make(double al, double be, double ga, uint32_t xfix) {
        return St13Coef{xfix & 1 ? 1.0 : al, xfix & 1 ? 0.0 : be, xfix & 1 ? 0.0 : ga,
                        xfix & 2 ? 1.0 : al, xfix & 2 ? 0.0 : be, xfix & 2 ? 0.0 : ga};
    }
};

// the window of a level: planes q-2 (M2), q-1 (M1), q (H), q+1 (P1); y-edge
// rows of H: two above (t2 farther, t1 nearer) and two below (b1 nearer, b2)
template <typename T, int VY> struct Win5 { const Bk<T, VY> &M2, &M1, &H, &P1; };

// Phase A.  fast: A = alpha*c + beta*((x1 + y1) + (zm1 + zp1)) + gamma*((x2 + y2) + zm2)
// exact: A = alpha*c (+) beta*S1 (the oracle's p + q), G = x2 + y2
template <int NTX, int VY, bool EXACT>
__device__ __forceinline__ void phaseA13(const Win5<float, VY>& w, const Rw<float>& t2, const Rw<float>& t1,
                                         const Rw<float>& b1, const Rw<float>& b2, const St13Coef<float>& k,
                                         Bk<float, VY>& A, Bk<float, VY>& G) {
    float2 L[VY], R[VY];
    xshfl2<NTX, VY>(w.H, L, R);
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        const Rw<float>& c = w.H.r[j];
        const Rw<float>& ym1 = j >= 1 ? w.H.r[j - 1] : t1;
        const Rw<float>& yp1 = j + 1 < VY ? w.H.r[j + 1] : b1;
        const Rw<float>& ym2 = j >= 2 ? w.H.r[j - 2] : (j == 1 ? t1 : t2);
        const Rw<float>& yp2 = j + 2 < VY ? w.H.r[j + 2] : (j + 2 == VY ? b1 : b2);
        // distance 1: (c0, c1) -> (L3 + c1, c0 + c2); (c2, c3) -> (c1 + c3, c2 + R0)
        const float2 x1a = __fadd2_rn(make_float2(c.a.y, c.a.x), make_float2(L[j].y, c.b.x));
        const float2 x1b = __fadd2_rn(make_float2(c.b.y, c.b.x), make_float2(c.a.y, R[j].x));
        // distance 2: (c0, c1) -> (L2 + c2, L3 + c3); (c2, c3) -> (c0 + R0, c1 + R1)
        const float2 x2a = __fadd2_rn(L[j], c.b);
        const float2 x2b = __fadd2_rn(c.a, R[j]);
        const float2 y1a = __fadd2_rn(ym1.a, yp1.a), y1b = __fadd2_rn(ym1.b, yp1.b);
        const float2 y2a = __fadd2_rn(ym2.a, yp2.a), y2b = __fadd2_rn(ym2.b, yp2.b);
        const float2 z1a = __fadd2_rn(w.M1.r[j].a, w.P1.r[j].a), z1b = __fadd2_rn(w.M1.r[j].b, w.P1.r[j].b);
        const float2 s1a = __fadd2_rn(__fadd2_rn(x1a, y1a), z1a), s1b = __fadd2_rn(__fadd2_rn(x1b, y1b), z1b);
        if (EXACT) {
            A.r[j].a = make_float2(__fadd_rn(__fmul_rn(k.alA.x, c.a.x), __fmul_rn(k.beA.x, s1a.x)),
                                   __fadd_rn(__fmul_rn(k.alA.y, c.a.y), __fmul_rn(k.beA.y, s1a.y)));
            A.r[j].b = make_float2(__fadd_rn(__fmul_rn(k.alB.x, c.b.x), __fmul_rn(k.beB.x, s1b.x)),
                                   __fadd_rn(__fmul_rn(k.alB.y, c.b.y), __fmul_rn(k.beB.y, s1b.y)));
            G.r[j].a = __fadd2_rn(x2a, y2a);
            G.r[j].b = __fadd2_rn(x2b, y2b);
        } else {
            const float2 s2a = __fadd2_rn(__fadd2_rn(x2a, y2a), w.M2.r[j].a);
            const float2 s2b = __fadd2_rn(__fadd2_rn(x2b, y2b), w.M2.r[j].b);
            A.r[j].a = __ffma2_rn(k.gaA, s2a, __ffma2_rn(k.beA, s1a, __fmul2_rn(k.alA, c.a)));
            A.r[j].b = __ffma2_rn(k.gaB, s2b, __ffma2_rn(k.beB, s1b, __fmul2_rn(k.alB, c.b)));
        }
    }
}
template <int NTX, int VY, bool EXACT>
__device__ __forceinline__ void phaseA13(const Win5<double, VY>& w, const Rw<double>& t2, const Rw<double>& t1,
                                         const Rw<double>& b1, const Rw<double>& b2, const St13Coef<double>& k,
                                         Bk<double, VY>& A, Bk<double, VY>& G) {
    double2 L[VY], R[VY];
    xshfl2<NTX, VY>(w.H, L, R);
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        const Rw<double>& c = w.H.r[j];
        const Rw<double>& ym1 = j >= 1 ? w.H.r[j - 1] : t1;
        const Rw<double>& yp1 = j + 1 < VY ? w.H.r[j + 1] : b1;
        const Rw<double>& ym2 = j >= 2 ? w.H.r[j - 2] : (j == 1 ? t1 : t2);
        const Rw<double>& yp2 = j + 2 < VY ? w.H.r[j + 2] : (j + 2 == VY ? b1 : b2);
        // (c0, c1): x-1 = (L1, c0), x+1 = (c1, R0), x-2 = (L0, L1), x+2 = (R0, R1)
        const double x10 = __dadd_rn(L[j].y, c.x1), x11 = __dadd_rn(c.x0, R[j].x);
        const double x20 = __dadd_rn(L[j].x, R[j].x), x21 = __dadd_rn(L[j].y, R[j].y);
        const double y10 = __dadd_rn(ym1.x0, yp1.x0), y11 = __dadd_rn(ym1.x1, yp1.x1);
        const double y20 = __dadd_rn(ym2.x0, yp2.x0), y21 = __dadd_rn(ym2.x1, yp2.x1);
        const double s10 = __dadd_rn(__dadd_rn(x10, y10), __dadd_rn(w.M1.r[j].x0, w.P1.r[j].x0));
        const double s11 = __dadd_rn(__dadd_rn(x11, y11), __dadd_rn(w.M1.r[j].x1, w.P1.r[j].x1));
        if (EXACT) {
            A.r[j].x0 = __dadd_rn(__dmul_rn(k.al0, c.x0), __dmul_rn(k.be0, s10));
            A.r[j].x1 = __dadd_rn(__dmul_rn(k.al1, c.x1), __dmul_rn(k.be1, s11));
            G.r[j].x0 = __dadd_rn(x20, y20);
            G.r[j].x1 = __dadd_rn(x21, y21);
        } else {
            const double s20 = __dadd_rn(__dadd_rn(x20, y20), w.M2.r[j].x0);
            const double s21 = __dadd_rn(__dadd_rn(x21, y21), w.M2.r[j].x1);
            A.r[j].x0 = __fma_rn(k.ga0, s20, __fma_rn(k.be0, s10, __dmul_rn(k.al0, c.x0)));
            A.r[j].x1 = __fma_rn(k.ga1, s21, __fma_rn(k.be1, s11, __dmul_rn(k.al1, c.x1)));
        }
    }
}

// Phase C: fast out = A + gamma*zp2; exact out = A (+) gamma*(G + (zm2 + zp2))
template <int VY, bool EXACT>
__device__ __forceinline__ void phaseC13(const Bk<float, VY>& A, const Bk<float, VY>& G, const Bk<float, VY>& M2,
                                         const Bk<float, VY>& F, const St13Coef<float>& k, Bk<float, VY>& O) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        if (EXACT) {
            const float2 sa = __fadd2_rn(G.r[j].a, __fadd2_rn(M2.r[j].a, F.r[j].a));
            const float2 sb = __fadd2_rn(G.r[j].b, __fadd2_rn(M2.r[j].b, F.r[j].b));
            O.r[j].a = make_float2(__fadd_rn(A.r[j].a.x, __fmul_rn(k.gaA.x, sa.x)), __fadd_rn(A.r[j].a.y, __fmul_rn(k.gaA.y, sa.y)));
            O.r[j].b = make_float2(__fadd_rn(A.r[j].b.x, __fmul_rn(k.gaB.x, sb.x)), __fadd_rn(A.r[j].b.y, __fmul_rn(k.gaB.y, sb.y)));
        } else {
            O.r[j].a = __ffma2_rn(k.gaA, F.r[j].a, A.r[j].a);
            O.r[j].b = __ffma2_rn(k.gaB, F.r[j].b, A.r[j].b);
        }
    }
}
template <int VY, bool EXACT>
__device__ __forceinline__ void phaseC13(const Bk<double, VY>& A, const Bk<double, VY>& G, const Bk<double, VY>& M2,
                                         const Bk<double, VY>& F, const St13Coef<double>& k, Bk<double, VY>& O) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        if (EXACT) {
            const double s0 = __dadd_rn(G.r[j].x0, __dadd_rn(M2.r[j].x0, F.r[j].x0));
            const double s1 = __dadd_rn(G.r[j].x1, __dadd_rn(M2.r[j].x1, F.r[j].x1));
            O.r[j].x0 = __dadd_rn(A.r[j].x0, __dmul_rn(k.ga0, s0));
            O.r[j].x1 = __dadd_rn(A.r[j].x1, __dmul_rn(k.ga1, s1));
        } else {
            O.r[j].x0 = __fma_rn(k.ga0, F.r[j].x0, A.r[j].x0);
            O.r[j].x1 = __fma_rn(k.ga1, F.r[j].x1, A.r[j].x1);
        }
    }
}

struct St13Params {
    St7Params g;       // geometry, work split, ring (alpha/beta in g)
    double gamma;
};

template <typename T, int D, int NTX, int VY, bool EXACT, int NT>
__global__ void __launch_bounds__(NT, 1)
st13_35d_kernel(const __grid_constant__ CUtensorMap tmap, const St13Params P) {
    constexpr int R = ST13_R;
    constexpr int RD = R * D;
    constexpr int VX = sizeof(T) == 4 ? 4 : 2;
    constexpr int TX = NTX * VX;
    constexpr int S = 2 * R + 1;   // window slots per level
    using V = typename std::conditional<sizeof(T) == 4, float4, double2>::type;
    using B = Bk<T, VY>;
    const St7Params& p = P.g;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    const int tid = threadIdx.x;
    const int NTH = blockDim.x;
    const int tx = tid % NTX;
    const int ty = tid / NTX;
    const int NTY = NTH / NTX;
    const int TY = NTY * VY;
    const T al = T(p.alpha), be = T(p.beta), ga = T(P.gamma);

    // ring of RING level-0 plane slots: round r reads planes r-2 (Y-edge rows of
    // level 1's centre) .. r; PF = RING-3 planes are in flight
    const int RING = p.ring, PF = p.ring - 3;
    const int slot_elems = TX * TY;
    const uint32_t slot_bytes = (uint32_t)(slot_elems * sizeof(T));
    T* ring = reinterpret_cast<T*>(smem_raw);
    // row exchange [level 1..D-1][round mod 3][N rows 0,1 / S rows 0,1][NTH] (16-byte rows)
    V* xbuf = reinterpret_cast<V*>(ring + RING * slot_elems);
    uint64_t* bars = reinterpret_cast<uint64_t*>(xbuf + (D > 1 ? (D - 1) * 3 * 4 * NTH : 0));

    for (int i = tid; i < RING * slot_elems * (int)sizeof(T) / 16; i += NTH)
        reinterpret_cast<float4*>(ring)[i] = make_float4(0.f, 0.f, 0.f, 0.f);
    fence_proxy_async();
    if (tid == 0) {
        prefetch_tensormap(&tmap);
        for (int s = 0; s < RING; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
    }
    __syncthreads();
    pdl_trigger();
    pdl_wait();

    B pl[D][S];
#pragma unroll
    for (int l = 0; l < D; ++l)
#pragma unroll
        for (int k = 0; k < S; ++k)
#pragma unroll
            for (int j = 0; j < VY; ++j) pl[l][k].r[j] = Rw<T>{};

    const int nzo = p.zb - p.za;
    int item = p.split[blockIdx.x];
    const int item_end = p.split[blockIdx.x + 1];
    const int zmin = max(0, -p.zbase);
    const int zmax = min(p.nzb - 1, p.nzg - 1 - p.zbase);
    const int my_off = (VY * ty) * TX + VX * tx;
    // y-edge rows of my block in a ring plane: 2 above, 2 below (clamped inside the tile)
    const int t2_off = max(VY * ty - 2, 0) * TX + VX * tx, t1_off = max(VY * ty - 1, 0) * TX + VX * tx;
    const int b1_off = min(VY * ty + VY, TY - 1) * TX + VX * tx, b2_off = min(VY * ty + VY + 1, TY - 1) * TX + VX * tx;
    const int tyu = max(ty - 1, 0), tyd = min(ty + 1, NTY - 1);
    const size_t plane = (size_t)p.nx * p.ny;
    uint32_t nload = 0;

    struct Seg { int tile, za, zb, rl0, rl1; };
    auto seg_at = [&](int it) {
        Seg g;
        g.tile = it / nzo;
        const int seg_end = min(item_end, (g.tile + 1) * nzo);
        g.za = p.za + (it - g.tile * nzo);
        g.zb = p.za + (seg_end - g.tile * nzo);
        g.rl0 = max(g.za - RD, zmin);
        g.rl1 = min(g.zb - 1 + RD, zmax);
        return g;
    };
    int pre = 0;

    while (item < item_end) {
        const Seg sg = seg_at(item);
        const int za = sg.za, zb = sg.zb, rl0 = sg.rl0, rl1 = sg.rl1;
        item += zb - za;
        const bool has_next = item < item_end;
        const Seg nx = seg_at(has_next ? item : item - 1);
        const St7Tile tl = st7_tile(p, sg.tile, RD);
        const St7Tile tn = st7_tile(p, nx.tile, RD);

        const int xg0 = tl.Lx + VX * tx;
        uint32_t xfix = 0, rowfix = 0, rowout = 0, rowmask = 0;
#pragma unroll
        for (int i = 0; i < VX; ++i)
            if (xg0 + i < R || xg0 + i >= p.nx - R) xfix |= 1u << i;
#pragma unroll
        for (int j = 0; j < VY; ++j) {
            const int yg = tl.Ly + VY * ty + j;
            if (yg >= tl.oy0 && yg < tl.oy1) rowmask |= 1u << j;
            if ((yg >= 0 && yg < R) || (yg >= p.ny - R && yg < p.ny)) rowfix |= 1u << j;
            if (yg < 0 || yg >= p.ny) rowout |= 1u << j;
        }
        const bool allfix = rowfix != 0 && (rowfix | rowout) == (1u << VY) - 1;
        const bool yslow = __any_sync(0xffffffffu, rowfix != 0 && !allfix);
        if (!(xg0 >= tl.ox0 && xg0 < tl.ox1)) rowmask = 0;
        const St13Coef<T> kc = St13Coef<T>::make(al, be, ga, allfix ? 0xFu : xfix);

        const int r0 = rl0, r1 = zb - 1 + RD;
        const int rs0 = max(max(za + RD, zmin + RD), -p.zbase + RD + R);
        const int rs1 = min(min(zb - 1 + RD, zmax + R), min(rl1, p.nzg - R - p.zbase + R - 1));
        T* pout = reinterpret_cast<T*>(p.out) + xg0 + (size_t)(tl.Ly + VY * ty) * p.nx +
                  (long long)(r0 - RD) * (long long)plane;
        const uint32_t kbase = nload;
        if (tid == 0) {
            for (int q = rl0 + pre; q <= min(rl0 + PF - 1, rl1); ++q) {
                const uint32_t k = (kbase + (q - rl0)) % RING;
                mbar_arrive_expect_tx(&bars[k], slot_bytes);
                tma_load_3d(ring + k * slot_elems, &tmap, &bars[k], tl.Lx, tl.Ly, q);
            }
            pre = 0;
        }
        nload = kbase + (uint32_t)max(0, rl1 - rl0 + 1);
        uint32_t slot_r = kbase % RING, par_r = (kbase / RING) & 1;
        uint32_t slot_f = (kbase + PF) % RING;
        uint32_t slot_m2 = (slot_r + RING - 2) % RING;   // plane r-2

        auto round = [&](auto PHc, auto STEADYc, int r) {
            constexpr int PH = decltype(PHc)::value;
            constexpr bool STEADY = decltype(STEADYc)::value;
            constexpr int sM2 = PH % S, sM1 = (PH + 1) % S, sH = (PH + 2) % S, sP1 = (PH + 3) % S, sN = (PH + 4) % S;
            const int r3 = r % 3;
            if (tid == 0) {
                if (r + PF <= rl1) {
                    mbar_arrive_expect_tx(&bars[slot_f], slot_bytes);
                    tma_load_3d(ring + slot_f * slot_elems, &tmap, &bars[slot_f], tl.Lx, tl.Ly, r + PF);
                } else if (has_next && pre < PF && pre == r + PF - rl1 - 1 && nx.rl0 + pre <= nx.rl1) {
                    mbar_arrive_expect_tx(&bars[slot_f], slot_bytes);
                    tma_load_3d(ring + slot_f * slot_elems, &tmap, &bars[slot_f], tn.Lx, tn.Ly, nx.rl0 + pre);
                    ++pre;
                }
            }
            bool zf[D + 1];
#pragma unroll
            for (int l = 1; l <= D; ++l) {
                zf[l] = false;
                if (!STEADY) {
                    const int zg = p.zbase + r - R * l;
                    zf[l] = zg < R || zg >= p.nzg - R;
                }
            }
            // ---- phase A
            B acc[D + 1], gs[EXACT ? D + 1 : 1];
#pragma unroll
            for (int l = 1; l <= D; ++l) {
                const int k = l - 1;
                Rw<T> t2, t1, b1, b2;
                if (l == 1) {   // level-0 plane r-2: neighbour rows from the ring
                    const T* sl = ring + slot_m2 * slot_elems;
                    t2 = ld_row(sl + t2_off); t1 = ld_row(sl + t1_off);
                    b1 = ld_row(sl + b1_off); b2 = ld_row(sl + b2_off);
                } else {        // rows level l-1 exchanged in round r-2
                    const V* xb = xbuf + ((l - 2) * 3 + (r3 + 1) % 3) * 4 * NTH;   // (r-2) mod 3
                    // the block above wrote its S rows (its rows VY-2, VY-1), the block below its N rows (0, 1)
                    t2 = ld_row(reinterpret_cast<const T*>(xb + 2 * NTH + tyu * NTX + tx));
                    t1 = ld_row(reinterpret_cast<const T*>(xb + 3 * NTH + tyu * NTX + tx));
                    b1 = ld_row(reinterpret_cast<const T*>(xb + 0 * NTH + tyd * NTX + tx));
                    b2 = ld_row(reinterpret_cast<const T*>(xb + 1 * NTH + tyd * NTX + tx));
                }
                const Win5<T, VY> w{pl[k][sM2], pl[k][sM1], pl[k][sH], pl[k][sP1]};
                phaseA13<NTX, VY, EXACT>(w, t2, t1, b1, b2, kc, acc[l], gs[EXACT ? l : 0]);
            }
            if (STEADY || r <= rl1) {
                mbar_wait(&bars[slot_r], par_r);
                const T* s0 = ring + slot_r * slot_elems + my_off;
#pragma unroll
                for (int j = 0; j < VY; ++j) pl[0][sN].r[j] = ld_row(s0 + j * TX);
            }
            // ---- phase C
#pragma unroll
            for (int l = 1; l <= D; ++l) {
                const int k = l - 1;
                B out;
                phaseC13<VY, EXACT>(acc[l], gs[EXACT ? l : 0], pl[k][sM2], pl[k][sN], kc, out);
                if (!STEADY) {
                    if (yslow) fix_rows(out, pl[k][sH], rowfix);
                    if (zf[l]) out = pl[k][sH];
                }
                if (l < D) {
                    pl[l < D ? l : 0][sN] = out;
                    T* xb = reinterpret_cast<T*>(xbuf + ((l - 1) * 3 + r3) * 4 * NTH + tid);
                    st_row(xb, out.r[0]);
                    st_row(xb + 1 * NTH * VX, out.r[VY > 1 ? 1 : 0]);
                    st_row(xb + 2 * NTH * VX, out.r[VY > 1 ? VY - 2 : 0]);
                    st_row(xb + 3 * NTH * VX, out.r[VY - 1]);
                } else if (STEADY || (r - RD >= za && r - RD < zb)) {
#pragma unroll
                    for (int j = 0; j < VY; ++j)
                        if (rowmask & (1u << j)) st_row(pout + j * p.nx, out.r[j]);
                }
            }
            __syncthreads();
            pout += plane;
            slot_m2 = (slot_m2 + 1 == (uint32_t)RING) ? 0 : slot_m2 + 1;
            if (++slot_r == (uint32_t)RING) { slot_r = 0; par_r ^= 1; }
            if (++slot_f == (uint32_t)RING) slot_f = 0;
        };
        using I0 = std::integral_constant<int, 0>;
        using I1 = std::integral_constant<int, 1>;
        using I2 = std::integral_constant<int, 2>;
        using I3 = std::integral_constant<int, 3>;
        using I4 = std::integral_constant<int, 4>;
        int r = r0, ph = 0;
        while (r <= r1) {
            if (ph == 0 && !yslow && r >= rs0 && r + 4 <= rs1) {
                do {
                    round(I0{}, std::true_type{}, r);
                    round(I1{}, std::true_type{}, r + 1);
                    round(I2{}, std::true_type{}, r + 2);
                    round(I3{}, std::true_type{}, r + 3);
                    round(I4{}, std::true_type{}, r + 4);
                    r += 5;
                } while (r + 4 <= rs1);
                continue;
            }
            switch (ph) {
                case 0: round(I0{}, std::false_type{}, r); break;
                case 1: round(I1{}, std::false_type{}, r); break;
                case 2: round(I2{}, std::false_type{}, r); break;
                case 3: round(I3{}, std::false_type{}, r); break;
                default: round(I4{}, std::false_type{}, r); break;
            }
            ++r;
            ph = ph == S - 1 ? 0 : ph + 1;
        }
    }
}

}  // namespace st35d
