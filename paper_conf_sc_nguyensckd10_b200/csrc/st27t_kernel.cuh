// st27t_kernel.cuh — 3.5D-blocked 27-point sweep on the 7-point machinery
// (PAPER.md P:119 defines the 27-point update, P:195-210 /
// P:251 the multi-level sweep; reading X24 for the weights).  Tolerance build.
//
// B = alpha*a + beta*F + gamma*E + delta*K over the 3x3x3 cube, with the
// plane-factorised sums of X24: for every plane of a level each point forms
//   v = a[y-1] + a[y+1], h = a[x-1] + a[x+1], f = h + v, e = v[x-1] + v[x+1]
// (f: the 4 in-plane face neighbours, e: the 4 in-plane corners), and
//   F = f(q) + a(q-1) + a(q+1), E = e(q) + f(q-1) + f(q+1), K = e(q-1) + e(q+1).
//
// Schedule.  The in-plane sums of a plane need its y neighbours, which a
// thread block only has after the row exchange of the round that produced
// the plane, so a level consumes the plane its lower level produced in the
// PREVIOUS round: level l at round r reads level l-1's plane p (level 0:
// plane r from the TMA ring, level l > 1: the plane level l-1 produced in
// round r-1) and
//   * completes its own plane q = p-1:  out = P(q) + beta*a(p) + gamma*f(p) + delta*e(p),
//   * starts plane p:  P(p) = alpha*a(p) + beta*(f(p) + a(p-1)) + gamma*(e(p) + f(p-1)) + delta*e(p-1),
// so a level carries (a, f, e) of its last input plane and the running partial
// P (4 values per point instead of the 9 of a three-plane window), its plane q
// is r - (2l - 1) (lag 2 per level beyond the first; the paper's z_s = z +
// 2R(dim_T - t')), and the levels of a round are independent: no serial
// chain inside a round, the level-1 work waits for the TMA plane last.
// The summation order differs from the oracle's (X24): tolerance build only
// (st27.cu keeps the oracle order for the bit-exact build).
//
// Mapping as the 7-point kernel: persistent CTAs over equal-cost (tile, z)
// work (split_work), TMA plane ring with per-slot mbarriers, a thread owns a
// 4-wide (FP32) / 2-wide (FP64) x VY block, X neighbours of the block edges by
// shuffle (one value per side for a and one for v: 4 shuffles per row), Y edge
// rows through a shared-memory exchange double-buffered by round parity,
// FP32 pairs as FADD2/FFMA2.  Shell points: x-shell columns and y-shell rows
// (planner y placement) get coefficients (1, 0, 0, 0), so out = P = a exactly;
// z-shell planes and unaligned y-shell rows are copied in checked rounds.
#pragma once
#include "st7_kernel.cuh"

namespace st35d {

// per-column coefficients; a fixed (shell) column gets (1, 0, 0, 0)
template <typename T> struct St27Coef;
template <> struct St27Coef<float> {
    float2 al[2], be[2], ga[2], de[2];   // [pair a = (c0, c1), pair b = (c2, c3)]
    static __device__ __forceinline__ St27Coef make(float al_, float be_, float ga_, float de_, uint32_t xfix) {
        St27Coef k;
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const bool f0 = xfix & (1u << (2 * h)), f1 = xfix & (2u << (2 * h));
            k.al[h] = make_float2(f0 ? 1.f : al_, f1 ? 1.f : al_);
            k.be[h] = make_float2(f0 ? 0.f : be_, f1 ? 0.f : be_);
            k.ga[h] = make_float2(f0 ? 0.f : ga_, f1 ? 0.f : ga_);
            k.de[h] = make_float2(f0 ? 0.f : de_, f1 ? 0.f : de_);
        }
        return k;
    }
};
template <> struct St27Coef<double> {
    double al[2], be[2], ga[2], de[2];   // [column 0, column 1]
    static __device__ __forceinline__ St27Coef make(double al_, double be_, double ga_, double de_, uint32_t xfix) {
        St27Coef k;
#pragma unroll
        for (int i = 0; i < 2; ++i) {
            const bool f = xfix & (1u << i);
            k.al[i] = f ? 1.0 : al_; k.be[i] = f ? 0.0 : be_; k.ga[i] = f ? 0.0 : ga_; k.de[i] = f ? 0.0 : de_;
        }
        return k;
    }
};

// in-plane sums of one block: f (faces) and e (corners) from the rows a, the
// rows above (top) / below (bot) the block, shuffles for the x edges
template <int NTX, int VY>
__device__ __forceinline__ void plane_sums(const Bk<float, VY>& a, const Rw<float>& top, const Rw<float>& bot,
                                           Bk<float, VY>& f, Bk<float, VY>& e) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        const Rw<float>& ym = j > 0 ? a.r[j - 1] : top;
        const Rw<float>& yp = j < VY - 1 ? a.r[j + 1] : bot;
        const Rw<float>& c = a.r[j];
        Rw<float> v;
        v.a = __fadd2_rn(ym.a, yp.a);
        v.b = __fadd2_rn(ym.b, yp.b);
        const float L = __shfl_up_sync(0xffffffffu, c.b.y, 1, NTX), R = __shfl_down_sync(0xffffffffu, c.a.x, 1, NTX);
        const float Lv = __shfl_up_sync(0xffffffffu, v.b.y, 1, NTX), Rv = __shfl_down_sync(0xffffffffu, v.a.x, 1, NTX);
        // (c0, c1) -> (L + c1, c0 + c2);  (c2, c3) -> (c1 + c3, c2 + R)
        const float2 ha = __fadd2_rn(make_float2(c.a.y, c.a.x), make_float2(L, c.b.x));
        const float2 hb = __fadd2_rn(make_float2(c.b.y, c.b.x), make_float2(c.a.y, R));
        f.r[j].a = __fadd2_rn(ha, v.a);
        f.r[j].b = __fadd2_rn(hb, v.b);
        e.r[j].a = __fadd2_rn(make_float2(v.a.y, v.a.x), make_float2(Lv, v.b.x));
        e.r[j].b = __fadd2_rn(make_float2(v.b.y, v.b.x), make_float2(v.a.y, Rv));
    }
}
template <int NTX, int VY>
__device__ __forceinline__ void plane_sums(const Bk<double, VY>& a, const Rw<double>& top, const Rw<double>& bot,
                                           Bk<double, VY>& f, Bk<double, VY>& e) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        const Rw<double>& ym = j > 0 ? a.r[j - 1] : top;
        const Rw<double>& yp = j < VY - 1 ? a.r[j + 1] : bot;
        const Rw<double>& c = a.r[j];
        const double v0 = ym.x0 + yp.x0, v1 = ym.x1 + yp.x1;
        const double L = __shfl_up_sync(0xffffffffu, c.x1, 1, NTX), R = __shfl_down_sync(0xffffffffu, c.x0, 1, NTX);
        const double Lv = __shfl_up_sync(0xffffffffu, v1, 1, NTX), Rv = __shfl_down_sync(0xffffffffu, v0, 1, NTX);
        f.r[j].x0 = (L + c.x1) + v0;
        f.r[j].x1 = (c.x0 + R) + v1;
        e.r[j].x0 = Lv + v1;
        e.r[j].x1 = v0 + Rv;
    }
}

// out = P + beta*a + gamma*f + delta*e (plane q complete);
// P' = alpha*a + beta*(f + ap) + gamma*(e + fp) + delta*ep (plane p started)
template <int VY>
__device__ __forceinline__ void complete_start(const St27Coef<float>& k, const Bk<float, VY>& a, const Bk<float, VY>& f,
                                               const Bk<float, VY>& e, const Bk<float, VY>& ap,
                                               const Bk<float, VY>& fp, const Bk<float, VY>& ep, Bk<float, VY>& P,
                                               Bk<float, VY>& out) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const float2 av = h ? a.r[j].b : a.r[j].a, fv = h ? f.r[j].b : f.r[j].a, ev = h ? e.r[j].b : e.r[j].a;
            float2& Pv = h ? P.r[j].b : P.r[j].a;
            float2& ov = h ? out.r[j].b : out.r[j].a;
            ov = __ffma2_rn(k.de[h], ev, __ffma2_rn(k.ga[h], fv, __ffma2_rn(k.be[h], av, Pv)));
            const float2 t1 = __fadd2_rn(fv, h ? ap.r[j].b : ap.r[j].a);
            const float2 t2 = __fadd2_rn(ev, h ? fp.r[j].b : fp.r[j].a);
            Pv = __ffma2_rn(k.de[h], h ? ep.r[j].b : ep.r[j].a,
                            __ffma2_rn(k.ga[h], t2, __ffma2_rn(k.be[h], t1, __fmul2_rn(k.al[h], av))));
        }
    }
}
template <int VY>
__device__ __forceinline__ void complete_start(const St27Coef<double>& k, const Bk<double, VY>& a,
                                               const Bk<double, VY>& f, const Bk<double, VY>& e,
                                               const Bk<double, VY>& ap, const Bk<double, VY>& fp,
                                               const Bk<double, VY>& ep, Bk<double, VY>& P, Bk<double, VY>& out) {
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        out.r[j].x0 = __fma_rn(k.de[0], e.r[j].x0, __fma_rn(k.ga[0], f.r[j].x0, __fma_rn(k.be[0], a.r[j].x0, P.r[j].x0)));
        out.r[j].x1 = __fma_rn(k.de[1], e.r[j].x1, __fma_rn(k.ga[1], f.r[j].x1, __fma_rn(k.be[1], a.r[j].x1, P.r[j].x1)));
        P.r[j].x0 = __fma_rn(k.de[0], ep.r[j].x0,
                             __fma_rn(k.ga[0], e.r[j].x0 + fp.r[j].x0,
                                      __fma_rn(k.be[0], f.r[j].x0 + ap.r[j].x0, k.al[0] * a.r[j].x0)));
        P.r[j].x1 = __fma_rn(k.de[1], ep.r[j].x1,
                             __fma_rn(k.ga[1], e.r[j].x1 + fp.r[j].x1,
                                      __fma_rn(k.be[1], f.r[j].x1 + ap.r[j].x1, k.al[1] * a.r[j].x1)));
    }
}

struct St27tParams {
    St7Params g;           // geometry, work split, ring (alpha/beta in g)
    double gamma, delta;
};

template <typename T, int D, int NTX, int VY, int NT>
__global__ void __launch_bounds__(NT, 1)
st27t_kernel(const __grid_constant__ CUtensorMap tmap, const St27tParams P27) {
    constexpr int VX = sizeof(T) == 4 ? 4 : 2;
    constexpr int TX = NTX * VX;
    using V = typename std::conditional<sizeof(T) == 4, float4, double2>::type;
    using B = Bk<T, VY>;
    const St7Params& p = P27.g;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    const int tid = threadIdx.x;
    const int NTH = blockDim.x;
    const int tx = tid % NTX, ty = tid / NTX;
    const int NTY = NTH / NTX;
    const int TY = NTY * VY;

    // ring of RING level-0 plane slots: round r reads plane r; PF = RING-2 in flight
    const int RING = p.ring, PF = p.ring - 2;
    const int slot_elems = TX * TY;
    const uint32_t slot_bytes = (uint32_t)(slot_elems * sizeof(T));
    T* ring = reinterpret_cast<T*>(smem_raw);
    // row exchange [level 1..D-1][round parity][N row / S row][NTH] (16-byte rows)
    V* xbuf = reinterpret_cast<V*>(ring + RING * slot_elems);
    uint64_t* bars = reinterpret_cast<uint64_t*>(xbuf + (D > 1 ? (D - 1) * 4 * NTH : 0));

    for (int i = tid; i < RING * slot_elems * (int)sizeof(T) / 16; i += NTH)
        reinterpret_cast<float4*>(ring)[i] = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int i = tid; i < (D > 1 ? (D - 1) * 4 * NTH : 0); i += NTH) {
        V z{};
        xbuf[i] = z;
    }
    fence_proxy_async();
    if (tid == 0) {
        prefetch_tensormap(&tmap);
        for (int s = 0; s < RING; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
    }
    __syncthreads();
    pdl_trigger();
    pdl_wait();

    // per level (index l-1): (a, f, e) of its input planes in two register sets
    // alternating with the round parity (set [ph]: this round's plane p, set
    // [ph^1]: plane p-1; no copies: the rounds are unrolled by two), and the
    // running partial P.  Level l writes its output plane straight into level
    // l+1's set for the next round.
    B a2[D][2], f2[D][2], e2[D][2], Pp[D];
#pragma unroll
    for (int l = 0; l < D; ++l)
#pragma unroll
        for (int j = 0; j < VY; ++j) {
            a2[l][0].r[j] = a2[l][1].r[j] = f2[l][0].r[j] = f2[l][1].r[j] = Rw<T>{};
            e2[l][0].r[j] = e2[l][1].r[j] = Pp[l].r[j] = Rw<T>{};
        }
    int ph = 0;   // register-set parity of the next round

    const int nzo = p.zb - p.za;
    int item = p.split[blockIdx.x];
    const int item_end = p.split[blockIdx.x + 1];
    const int zmin = max(0, -p.zbase);
    const int zmax = min(p.nzb - 1, p.nzg - 1 - p.zbase);
    const int my_off = (VY * ty) * TX + VX * tx;
    const int top_off = max(VY * ty - 1, 0) * TX + VX * tx;
    const int bot_off = min(VY * ty + VY, TY - 1) * TX + VX * tx;
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
        g.rl0 = max(g.za - D, zmin);
        g.rl1 = min(g.zb - 1 + D, zmax);
        return g;
    };
    int pre = 0;

    while (item < item_end) {
        const Seg sg = seg_at(item);
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
        const bool allfix = rowfix != 0 && (rowfix | rowout) == (1u << VY) - 1;
        const bool yslow = __any_sync(0xffffffffu, rowfix != 0 && !allfix);   // warp-uniform
        if (!(xg0 >= tl.ox0 && xg0 < tl.ox1)) rowmask = 0;
        const St27Coef<T> kc = St27Coef<T>::make(T(p.alpha), T(p.beta), T(P27.gamma), T(P27.delta),
                                                 allfix ? 0xFu : xfix);

        // level D completes plane r - (2D - 1): rounds rl0 .. zb - 1 + 2D - 1
        constexpr int LAGD = 2 * D - 1;
        const int r0 = rl0, r1 = zb - 1 + LAGD;
        T* pout = reinterpret_cast<T*>(p.out) + xg0 + (size_t)(tl.Ly + VY * ty) * p.nx +
                  (long long)(r0 - LAGD) * (long long)plane;
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

        auto round = [&](auto PHc, auto STEADYc, int r) {
            constexpr int CU = decltype(PHc)::value, PV = CU ^ 1;
            constexpr bool STEADY = decltype(STEADYc)::value;
            const int rpar = r & 1;
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
            // one level: input plane a (+ y edge rows), complete plane q = p-1, start p
            auto level = [&](auto Lc, const Rw<T>& top, const Rw<T>& bot) {
                constexpr int l = decltype(Lc)::value;
                constexpr int k = l - 1;
                B out;
                plane_sums<NTX, VY>(a2[k][CU], top, bot, f2[k][CU], e2[k][CU]);
                complete_start<VY>(kc, a2[k][CU], f2[k][CU], e2[k][CU], a2[k][PV], f2[k][PV], e2[k][PV], Pp[k], out);
                if (!STEADY) {
                    const int zq = p.zbase + r - (2 * l - 1);   // global plane of the completed q
                    if (yslow) fix_rows(out, a2[k][PV], rowfix);
                    if (zq == 0 || zq == p.nzg - 1) out = a2[k][PV];   // z shell: a(q) unchanged
                }
                if constexpr (l < D) {
                    a2[l][PV] = out;   // level l+1's input in round r+1 (read as set PV before: levels descend)
                    T* xb = reinterpret_cast<T*>(xbuf + ((l - 1) * 4 + rpar * 2) * NTH + tid);
                    st_row(xb, out.r[0]);
                    st_row(xb + NTH * VX, out.r[VY - 1]);
                } else if (STEADY || (r - LAGD >= za && r - LAGD < zb)) {
#pragma unroll
                    for (int j = 0; j < VY; ++j)
                        if (rowmask & (1u << j)) st_row(pout + j * p.nx, out.r[j]);
                }
            };
            // levels D .. 2 first (their inputs are last round's planes), level 1 last
            static_for<0, D - 1>([&](auto Ic) {
                constexpr int l = D - decltype(Ic)::value;   // D, D-1, ..., 2
                const V* xb = xbuf + ((l - 2) * 4 + (rpar ^ 1) * 2) * NTH;   // written by level l-1 in round r-1
                const Rw<T> top = ld_row(reinterpret_cast<const T*>(xb + NTH + tyu * NTX + tx));
                const Rw<T> bot = ld_row(reinterpret_cast<const T*>(xb + tyd * NTX + tx));
                level(std::integral_constant<int, l>{}, top, bot);
            });
            {
                Rw<T> top, bot;
                if (STEADY || r <= rl1) {
                    mbar_wait(&bars[slot_r], par_r);
                    const T* sl = ring + slot_r * slot_elems;
#pragma unroll
                    for (int j = 0; j < VY; ++j) a2[0][CU].r[j] = ld_row(sl + my_off + j * TX);
                    top = ld_row(sl + top_off);
                    bot = ld_row(sl + bot_off);
                } else {   // past the last level-0 plane: stale values, never stored
                    top = a2[0][CU].r[0];
                    bot = a2[0][CU].r[VY - 1];
                }
                level(std::integral_constant<int, 1>{}, top, bot);
            }
            __syncthreads();
            pout += plane;
            if (++slot_r == (uint32_t)RING) { slot_r = 0; par_r ^= 1; }
            if (++slot_f == (uint32_t)RING) slot_f = 0;
        };
        // steady rounds: the level-0 plane exists, the output plane is in the
        // segment, and no level completes a z-shell plane; no unaligned y-shell row
        const int rs0 = max(za + LAGD, -p.zbase + LAGD + 1);
        const int rs1 = min(min(zb - 1 + LAGD, rl1), p.nzg - 1 - p.zbase);
        using I0 = std::integral_constant<int, 0>;
        using I1 = std::integral_constant<int, 1>;
        using ST = std::true_type;
        using CK = std::false_type;
        int r = r0;
        while (r <= r1) {
            const bool st = !yslow && r >= rs0 && r <= rs1;
            if (st && r + 1 <= rs1) {   // two steady rounds: the parity returns to ph
                if (ph == 0) { round(I0{}, ST{}, r); round(I1{}, ST{}, r + 1); }
                else { round(I1{}, ST{}, r); round(I0{}, ST{}, r + 1); }
                r += 2;
                continue;
            }
            if (ph == 0) { if (st) round(I0{}, ST{}, r); else round(I0{}, CK{}, r); }
            else { if (st) round(I1{}, ST{}, r); else round(I1{}, CK{}, r); }
            ph ^= 1;
            ++r;
        }
    }
}

}  // namespace st35d
