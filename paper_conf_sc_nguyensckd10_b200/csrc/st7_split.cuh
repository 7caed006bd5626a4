// st7_split.cuh — warp-specialised variant of the 3.5D 7-point sweep.
//
// The register Z windows of st7_35d_kernel (3 planes x 16 values per level
// and thread) cap the CTA at ~8 warps per SM, and the kernel is then latency
// bound.  Here the dim_T levels are split between two thread groups that own
// the SAME tile blocks: group A (first half of the threads) computes levels
// 1..DA from the TMA ring, group B (second half) levels DA+1..D from a
// 4-plane shared-memory hand-off ring that group A fills with its level-DA
// planes.  Each thread keeps the Z windows of only its own group's levels, so
// twice the warps fit.  Group B runs one round behind group A (it consumes
// hand-off planes written in earlier rounds), so one CTA barrier per round
// still suffices.  Arithmetic and operation order are st7_level's.
#pragma once
#include "st7_kernel.cuh"

namespace st35d {

__device__ __forceinline__ void cta_bar() { asm volatile("bar.sync 0;" ::: "memory"); }

template <typename T, int D, int DA, int NTX, int VY, bool EXACT, int MAXT>
__global__ void __launch_bounds__(MAXT, 1)
st7_35d_split_kernel(const __grid_constant__ CUtensorMap tmap, const St7Params p) {
    static_assert(DA >= 1 && DA < D, "split point");
    constexpr int VX = Vec<T>::N;
    constexpr int TX = NTX * VX;
    constexpr int GM = MAXT / 2;                    // max threads per group
    using V = typename Vec<T>::type;
    using B = Blk<T, VY>;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    const int GT = blockDim.x / 2;
    const int tid = threadIdx.x;
    const bool grpB = tid >= GT;
    const int gtid = grpB ? tid - GT : tid;
    const int tx = gtid % NTX, ty = gtid / NTX;
    const int NTY = GT / NTX;
    const int TY = NTY * VY;
    const T al = T(p.alpha), be = T(p.beta);

    const int RING = p.ring, PF = p.ring - 3;
    const int slot_elems = TX * TY;
    T* ring = reinterpret_cast<T*>(smem_raw);       // [RING][TY][TX]  level 0 (TMA)
    T* hand = ring + RING * slot_elems;             // [4][TY][TX]     level DA (group A -> B)
    V* xbuf = reinterpret_cast<V*>(hand + 4 * slot_elems);   // [D-2][2 parity][2 N/S][GM]
    uint64_t* bars = reinterpret_cast<uint64_t*>(xbuf + (D > 2 ? (D - 2) * 4 * GM : 0));

    for (int i = tid; i < (RING + 4) * slot_elems; i += blockDim.x) ring[i] = T(0);
    fence_proxy_async();
    if (tid == 0) {
        prefetch_tensormap(&tmap);
        for (int s = 0; s < RING; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
    }
    __syncthreads();

    const int nzo = p.zb - p.za;
    const long long item0 = p.split[blockIdx.x];
    const long long item_end = p.split[blockIdx.x + 1];
    const int zmin = max(0, -p.zbase);
    const int zmax = min(p.nzb - 1, p.nzg - 1 - p.zbase);
    const uint32_t tile_bytes = (uint32_t)(slot_elems * sizeof(T));

    const int tyu = max(ty - 1, 0), tyd = min(ty + 1, NTY - 1);
    const int my_off = (VY * ty) * TX + VX * tx;
    const int top_off = max(VY * ty - 1, 0) * TX + VX * tx;
    const int bot_off = min(VY * ty + VY, TY - 1) * TX + VX * tx;
    // exchange rows of in-register levels: A levels 1..DA-1 -> x = l-1, B levels DA+1..D-1 -> x = l-2
    V* const xw = xbuf + gtid;
    const V* const xtop = xbuf + GM + tyu * NTX + tx;
    const V* const xbot = xbuf + tyd * NTX + tx;
    T* outp = reinterpret_cast<T*>(p.out);
    const int nxs = p.nx;
    const size_t plane = (size_t)p.nx * p.ny;

    // Each group runs its own copy of the segment loop (same number of barriers
    // per segment), so only its own levels' register windows are live in it.
    auto run = [&](auto GRPc) {
        constexpr bool GB = decltype(GRPc)::value;
        constexpr int L0 = GB ? DA + 1 : 1, L1 = GB ? D : DA;     // this group's levels
        B pl[D][3];      // windows of in-register levels (L0..L1-1 minus the hand-off level)
        B outv;
#pragma unroll
        for (int l = L0; l < L1; ++l)
#pragma unroll
            for (int k = 0; k < 3; ++k) pl[l][k] = B{};
        long long item = item0;
        uint32_t nload = 0;
        while (item < item_end) {
            const int tile = (int)(item / nzo);
            const long long seg_end = min(item_end, (long long)(tile + 1) * nzo);
            const int za = p.za + (int)(item - (long long)tile * nzo);
            const int zb = p.za + (int)(seg_end - (long long)tile * nzo);
            item = seg_end;

            const int ix = tile % p.tiles_x, iy = tile / p.tiles_x;
            const int ox0 = ix * p.wx, ox1 = min(ox0 + p.wx, p.nx);
            const int oy0 = iy * p.wy, oy1 = min(oy0 + p.wy, p.ny);
            const int Lx = ox0 - p.hx;
            const int Ly = oy0 - D;
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
            if (!(xg0 >= ox0 && xg0 < ox1)) rowmask = 0;
            const Coef<T> kc = Coef<T>::make(al, be, xfix);
            const Coef<T> kf = Coef<T>::fixed();

            const int rl0 = max(za - D, zmin);
            const int rl1 = min(zb - 1 + D, zmax);
            const int r0 = rl0;
            const int r1 = zb - 1 + D;               // group A's last round; group B's is r1 + 1
            const uint32_t kbase = nload;
            nload = kbase + (uint32_t)max(0, rl1 - rl0 + 1);
            uint32_t slot_r = kbase % RING, par_r = (kbase / RING) & 1;
            uint32_t slot_f = (kbase + PF) % RING;
            uint32_t slot_m1 = (slot_r + RING - 1) % RING;
            uint32_t slot_m2 = (slot_r + RING - 2) % RING;
            if (!GB && tid == 0) {
                for (int q = rl0; q <= min(rl0 + PF - 1, rl1); ++q) {
                    const uint32_t k = kbase + (q - rl0);
                    uint64_t* bar = &bars[k % RING];
                    mbar_arrive_expect_tx(bar, tile_bytes);
                    tma_load_3d(ring + (k % RING) * slot_elems, &tmap, bar, Lx, Ly, q);
                }
            }
            // group B: level D at virtual round rb = r - 1 writes plane rb - D
            T* pout = outp + xg0 + (size_t)(Ly + VY * ty) * p.nx + (long long)(r0 - 1 - D) * (long long)plane;

            // level l at plane z from three full planes in shared memory (ring or hand-off)
            auto from_smem = [&](const T* s2, const T* s1, const T* s0, int z, B& dst) {
                const int zg = p.zbase + z;
                const bool zfix = (zg == 0) || (zg == p.nzg - 1);
                B zm, c, zp;
#pragma unroll
                for (int j = 0; j < VY; ++j) {
                    zm.load_nat(j, s2 + my_off + j * TX);
                    c.load_nat(j, s1 + my_off + j * TX);
                    zp.load_nat(j, s0 + my_off + j * TX);
                }
                const Row<T> top = row_nat(s1 + top_off), bot = row_nat(s1 + bot_off);
                st7_level<NTX, VY, EXACT>(zm, c, zp, top, bot, Coef<T>::sel(zfix, kf, kc), yslow, rowfix, dst);
            };

            auto round = [&](auto PHc, int r) {
                constexpr int PH = decltype(PHc)::value;
                constexpr int PREV = PH % 3, CUR = (PH + 1) % 3, NEW = (PH + 2) % 3;
                const int rv = GB ? r - 1 : r;            // this group's virtual round
                bool active = GB ? rv >= r0 : r <= r1;
                if (!GB && active) {
                    if (tid == 0 && r + PF <= rl1) {
                        uint64_t* bar = &bars[slot_f];
                        mbar_arrive_expect_tx(bar, tile_bytes);
                        tma_load_3d(ring + slot_f * slot_elems, &tmap, bar, Lx, Ly, r + PF);
                    }
                    if (r <= rl1) mbar_wait(&bars[slot_r], par_r);
                }
                if (p.dbg & 1) active = false;
                if (active) {
#pragma unroll
                    for (int l = L0; l <= L1; ++l) {
                        const int z = rv - l;
                        const int lo = max(za - (D - l), zmin), hi = min(zb - 1 + (D - l), zmax);
                        if (z < lo || z > hi) continue;
                        B& dst = (l == L1) ? outv : pl[l < D ? l : 1][NEW];
                        if (l == L0) {
                            if (!GB)
                                from_smem(ring + slot_m2 * slot_elems, ring + slot_m1 * slot_elems,
                                          ring + slot_r * slot_elems, z, dst);
                            else
                                from_smem(hand + (size_t)((z - 1) & 3) * slot_elems, hand + (size_t)(z & 3) * slot_elems,
                                          hand + (size_t)((z + 1) & 3) * slot_elems, z, dst);
                        } else {
                            const int zg = p.zbase + z;
                            const bool zfix = (zg == 0) || (zg == p.nzg - 1);
                            const int xin = GB ? l - 3 : l - 2;   // exchange rows of level l-1
                            const int o = (xin * 4 + (z & 1) * 2) * GM;
                            const Row<T> top = row_x(xtop + o), bot = row_x(xbot + o);
                            const int lp = l > 1 ? l - 1 : 1;
                            st7_level<NTX, VY, EXACT>(pl[lp][PREV], pl[lp][CUR], pl[lp][NEW], top, bot,
                                                      Coef<T>::sel(zfix, kf, kc), yslow, rowfix, dst);
                        }
                        if (l < L1) {                            // in-register level: exchange rows
                            const int xo = GB ? l - 2 : l - 1;
                            V* xb = xw + (xo * 4 + (z & 1) * 2) * GM;
                            dst.store_x(0, xb);
                            dst.store_x(VY - 1, xb + GM);
                        } else if (!GB) {                        // level DA: hand-off plane
                            T* h = hand + (size_t)(z & 3) * slot_elems + my_off;
#pragma unroll
                            for (int j = 0; j < VY; ++j) outv.store_x(j, reinterpret_cast<V*>(h + j * TX));
                        } else {                                 // level D: output
#pragma unroll
                            for (int j = 0; j < VY; ++j)
                                if (rowmask & (1u << j)) outv.store_global(j, pout + j * nxs);
                        }
                    }
                }
                if (!GB) {
                    slot_m2 = slot_m1;
                    slot_m1 = slot_r;
                    if (++slot_r == (uint32_t)RING) { slot_r = 0; par_r ^= 1; }
                    if (++slot_f == (uint32_t)RING) slot_f = 0;
                } else {
                    pout += plane;
                }
                cta_bar();
            };

            for (int r = r0; r <= r1 + 1;) {
                round(std::integral_constant<int, 0>{}, r);
                if (++r > r1 + 1) break;
                round(std::integral_constant<int, 1>{}, r);
                if (++r > r1 + 1) break;
                round(std::integral_constant<int, 2>{}, r);
                ++r;
            }
        }
    };
    if (!grpB) run(std::false_type{});
    else run(std::true_type{});
}

}  // namespace st35d
