// lbm_tma.cu — the D3Q19 pull pass of the gather form fed by TMA.
//
// Gather form (lbm_kernel.cuh): T push steps are P^T = S.(C.S)^(T-1).C, so the
// hot pass is the pull step C.S on the post-collision state g: for a FLUID
// cell x, f_i(x) = g_i(x - e_i) (P:125-129 streaming, read from the upstream
// neighbour), with half-way bounce-back g_opp(i)(x) [- (6 w e.u_lid)_opp(i)]
// when x - e_i is WALL [LID] (X10); then collide (X9) and store the 19 values
// at x.  Non-FLUID cells keep their values.
//
// B200 data movement (what the plain lbm_gather_kernel does with 19 shifted
// per-thread loads): a CTA streams XY tiles of BX x BY cells of one plane.  A
// producer warp issues, per tile, 19 TMA box loads from the lattice seen as a
// 3D tensor (x, y, 19 nz) — population i's box starts at row y0 - ey_i of plane
// i nz + z - ez_i: the y and z shifts of the stream are done by the TMA engine
// (out-of-lattice rows zero-filled).  A box start must be 16-byte aligned in x
// (measured: an x-shifted start faults with an illegal instruction), so the 10
// populations with ex = +-1 load a box A = 16 B wider on their upstream side and
// the consumer reads column cx - ex_i of it; the other 9 load the tile itself.  Tiles pass through an S-stage
// ring (full barrier: TMA transaction bytes; empty barrier: one arrive per
// consumer thread), so S-1 tiles of loads are always in flight.  Consumers read
// their 19 values from shared memory (conflict-free, consecutive cells), free
// the stage, collide in registers and write the 19 results with coalesced,
// aligned 128-byte-per-warp stores at the cell itself (the gather form's
// aligned stores).  Tiles of the first and last plane (all non-FLUID:
// the shell is checked) load unshifted boxes and are copied through; the
// collide-only first pass loads unshifted boxes everywhere, the stream-only
// last pass skips the collision.
#include "launch.h"


namespace st35d {

// tile of BX x BY = 256 cells (one per consumer thread), x halo A = 16 bytes;
// a TMA destination must be 128-byte aligned, so population slots are rounded up
template <typename T, int BX_> struct PullTile {
    static constexpr int BX = BX_, BY = 256 / BX_, A = 16 / (int)sizeof(T);
    static constexpr int SLOT = ((BX + A) * BY * (int)sizeof(T) + 127) / 128 * 128 / (int)sizeof(T);
};

constexpr int PULL_CONSUMERS = 256;   // consumer threads, one cell each per tile
constexpr int PULL_THREADS = PULL_CONSUMERS + 32;

// population i's box: width BX (ex = 0) or BX + A (ex = +-1: the 16-byte x halo
// on the upstream side), row pitch = box width; cell column cx reads column
// col0 + cx of the box
template <typename G, int I> struct PullBox {
    static constexpr int BX = G::BX, A = G::A;
    static constexpr int ex = D3Q19<I>::ex;
    static constexpr int pitch = ex == 0 ? BX : BX + A;
    static constexpr int xoff = ex > 0 ? -A : 0;          // box start relative to x0
    static constexpr int col0 = ex > 0 ? A - 1 : (ex < 0 ? 1 : 0);
};

// MODE (lbm_kernel.cuh): LBM_PULL = stream + collide (the hot pass), LBM_COLLIDE =
// collide only (unshifted boxes; may run in place, src == dst), LBM_STREAM =
// stream only.  The first and last pass of the gather form run the same kernel.
template <typename T, bool E, int MODE, int TBX>
__global__ void __launch_bounds__(PULL_THREADS, 2)
lbm_pull_tma_kernel(const __grid_constant__ CUtensorMap mapn, const __grid_constant__ CUtensorMap mapw,
                    const T* src, T* dst, const uint8_t* __restrict__ fl2, const LbmParams p,
                    int stages, int tiles_x, int tiles_y) {
    using G = PullTile<T, TBX>;
    constexpr int BX = G::BX, BY = G::BY, A = G::A, NC = PULL_CONSUMERS;
    static_assert(NC == BX * BY, "one consumer thread per tile cell");
    constexpr int SLOT = G::SLOT;                 // elements reserved per population box (128-byte aligned)
    constexpr uint32_t NB = BX * BY * sizeof(T), WB = (BX + A) * BY * sizeof(T);
    constexpr uint32_t TX_INTERIOR = 9 * NB + 10 * WB, TX_SHELL = 19 * NB;   // 9 populations with ex = 0
    extern __shared__ __align__(128) unsigned char smem_raw[];
    T* buf = reinterpret_cast<T*>(smem_raw);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw + (size_t)stages * 19 * SLOT * sizeof(T));
    uint64_t* empty = full + stages;

    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int s = 0; s < stages; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], NC); }
        fence_mbar_init();
    }
    __syncthreads();
    pdl_trigger();
    pdl_wait();   // the previous pass's writes are visible from here on

    // buffer planes [za, zb) (Z slabs: the owned planes or a part of them; the
    // buffer holds nz = nzb planes, global plane = zbase + buffer plane)
    const int nx = p.nx, ny = p.ny, nz = p.nzb, za = p.za;
    const int zs0 = -p.zbase, zs1 = p.nzg - 1 - p.zbase;   // buffer planes of the global z shell
    // tiles dealt round-robin (x fastest): at any moment the CTAs stream
    // neighbouring tiles of the same planes, so each population's rows are read
    // in address order across the chip and a tile's x halo is its neighbour's
    // edge, fetched by the next CTA at the same time (measured: contiguous tile
    // ranges per CTA scatter the reads over the lattice, 17 vs 26 GLUPS)
    const long long ntiles = (long long)tiles_x * tiles_y * (p.zb - p.za);
    const long long t_begin = blockIdx.x, t_end = ntiles, t_step = gridDim.x;
    auto where = [&](long long tile, int& x0, int& y0, int& z) {
        const int tx = (int)(tile % tiles_x);
        const long long r = tile / tiles_x;
        x0 = tx * BX; y0 = (int)(r % tiles_y) * BY; z = za + (int)(r / tiles_y);
    };
    if (tid >= NC) {   // producer warp: one lane issues the TMA loads
        if (tid == NC) {
            prefetch_tensormap(&mapn);
            prefetch_tensormap(&mapw);
            int k = 0;
            for (long long tile = t_begin; tile < t_end; tile += t_step, ++k) {
                const int s = k % stages;
                if (k >= stages) mbar_wait(&empty[s], ((k / stages) - 1) & 1);
                int x0, y0, z;
                where(tile, x0, y0, z);
                // shell planes (copied through) and the collide pass: own (unshifted) values
                const bool own = MODE == LBM_COLLIDE || z == zs0 || z == zs1;
                T* b = buf + (size_t)s * 19 * SLOT;
                if (own) {
                    mbar_arrive_expect_tx(&full[s], TX_SHELL);
                    for (int i = 0; i < 19; ++i) tma_load_3d(b + i * SLOT, &mapn, &full[s], x0, y0, i * nz + z);
                } else {
                    // population i's planes are planes i*nz .. i*nz+nz-1 of the 3D maps; interior
                    // planes shift by at most one plane, so a box never leaves its population
                    mbar_arrive_expect_tx(&full[s], TX_INTERIOR);
                    [&]<int... Is>(std::integer_sequence<int, Is...>) {
                        ((tma_load_3d(b + Is * SLOT, D3Q19<Is>::ex == 0 ? &mapn : &mapw, &full[s],
                                      x0 + PullBox<G, Is>::xoff, y0 - D3Q19<Is>::ey, Is * nz + z - D3Q19<Is>::ez)),
                         ...);
                    }(std::make_integer_sequence<int, 19>{});
                }
            }
        }
        return;
    }

    const size_t plane = (size_t)nx * ny;
    const size_t nc = plane * nz;
    const T omega = T(p.omega);
    const int cx = tid % BX, cy = tid / BX;
    // the cell's flag is read one tile ahead (its latency off the tile's critical path)
    auto flag_of = [&](long long tile) -> uint32_t {
        int x0, y0, z;
        where(tile, x0, y0, z);
        const int x = x0 + cx, y = y0 + cy;
        return x < nx && y < ny ? (uint32_t)fl2[(size_t)z * plane + (size_t)y * nx + x] : 0u;
    };
    uint32_t fl_next = t_begin < t_end ? flag_of(t_begin) : 0u;
    int k = 0;
    for (long long tile = t_begin; tile < t_end; tile += t_step, ++k) {
        const int s = k % stages;
        int x0, y0, z;
        where(tile, x0, y0, z);
        const uint32_t fl = fl_next;
        if (tile + t_step < t_end) fl_next = flag_of(tile + t_step);
        const bool own = MODE == LBM_COLLIDE || z == zs0 || z == zs1;   // unshifted boxes
        const int x = x0 + cx, y = y0 + cy;
        const bool inb = x < nx && y < ny;
        const size_t c = (size_t)z * plane + (size_t)y * nx + x;
        mbar_wait(&full[s], (k / stages) & 1);
        const T* b = buf + (size_t)s * 19 * SLOT;
        T f[19];
        if (own) {
#pragma unroll
            for (int i = 0; i < 19; ++i) f[i] = b[i * SLOT + cy * BX + cx];
        } else {
            [&]<int... Is>(std::integer_sequence<int, Is...>) {
                ((f[Is] = b[Is * SLOT + cy * PullBox<G, Is>::pitch + PullBox<G, Is>::col0 + cx]), ...);
            }(std::make_integer_sequence<int, 19>{});
        }
        // every consumer thread releases the stage itself, behind a generic->async
        // proxy fence: the stage is next written by TMA (async proxy), and the
        // thread's shared-memory reads (generic proxy) must be complete first.
        // Measured on B200 without the fence (release-semantics arrive alone, or one
        // arrive per warp after __syncwarp): the next TMA write overtook reads still
        // in flight — wrong cells on 256^3 FP64 with 2 CTAs per SM.
        fence_proxy_async();
        mbar_arrive(&empty[s]);
        if (!inb) continue;
        if (fl & 0x7fu) {   // WALL / LID: copied through (own values; unshifted tiles already hold them)
            if (!own) {
#pragma unroll
                for (int i = 0; i < 19; ++i) f[i] = src[(size_t)i * nc + c];
            }
        } else {
            if (!own && (fl & 0x80u)) {   // a non-FLUID upstream neighbour: half-way bounce-back (X10)
                // the 18 upstream flags and the cell's own 18 values are loaded together
                // (one memory round trip), then selected
                uint32_t sf[19];
                T mine[19];
                [&]<int... Is>(std::integer_sequence<int, Is...>) {
                    ((sf[Is] = Is == 0 ? 0u
                                       : (uint32_t)__ldg(fl2 + (long long)c -
                                                         ((long long)D3Q19<Is>::ex + (long long)D3Q19<Is>::ey * nx +
                                                          (long long)D3Q19<Is>::ez * (long long)plane))),
                     ...);
                    ((mine[Is] = Is == 0 ? T(0) : src[(size_t)D3Q19<Is>::opp * nc + c]), ...);
                }(std::make_integer_sequence<int, 19>{});
                auto bb = [&](auto Ic) {
                    constexpr int I = decltype(Ic)::value;
                    if constexpr (I > 0) {
                        const uint32_t t = sf[I] & 0x7fu;
                        if (t == 1) f[I] = mine[I];
                        else if (t != 0) f[I] = Ar<T, E>::sub(mine[I], T(p.lidc[D3Q19<I>::opp]));
                    }
                };
                [&]<int... Is>(std::integer_sequence<int, Is...>) { (bb(std::integral_constant<int, Is>{}), ...); }
                (std::make_integer_sequence<int, 19>{});
            }
            if (MODE != LBM_STREAM) collide<T, E>(f, omega);
        }
        T* d = dst + c;
#pragma unroll
        for (int i = 0; i < 19; ++i) d[(size_t)i * nc] = f[i];
    }
}

// tile width for a lattice row of nx cells (measured on B200, FP32 cavity, GLUPS,
// 64 x 4 vs 128 x 2 tiles: 256^3 34.1 / 30.8, 384^3 31.6 / 31.5, 512^3 35.0 / 32.9,
// 640^3 31.2 / 33.4, 1024^3 25.0 / 30.6)
static int pull_bx(int dtype, int nx) { return dtype == 0 ? (nx > 512 ? 128 : 64) : 32; }

template <typename T, int BX>
static size_t stage_bytes() { return 19u * PullTile<T, BX>::SLOT * sizeof(T); }

template <typename T, bool E, int BX>
static cudaError_t pull_t(int mode, bool pdl, const CUtensorMap* maps, const void* src, void* dst,
                          const uint8_t* fl2, const LbmParams& p, int grid, int stages, cudaStream_t s) {
    auto k = mode == LBM_COLLIDE ? lbm_pull_tma_kernel<T, E, LBM_COLLIDE, BX>
           : mode == LBM_STREAM  ? lbm_pull_tma_kernel<T, E, LBM_STREAM, BX> : lbm_pull_tma_kernel<T, E, LBM_PULL, BX>;
    const size_t smem = (size_t)stages * (stage_bytes<T, BX>() + 16);
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const int tiles_x = (p.nx + PullTile<T, BX>::BX - 1) / PullTile<T, BX>::BX;
    const int tiles_y = (p.ny + PullTile<T, BX>::BY - 1) / PullTile<T, BX>::BY;
    return launch_pdl(pdl, k, grid, PULL_THREADS, smem, s, maps[0], maps[1], static_cast<const T*>(src),
                      static_cast<T*>(dst), fl2, p, stages, tiles_x, tiles_y);
}

size_t lbm_pull_tma_stage_bytes(int dtype, int nx) {
    const int bx = pull_bx(dtype, nx);
    return (dtype == 1 ? stage_bytes<double, 32>() : bx == 128 ? stage_bytes<float, 128>() : stage_bytes<float, 64>())
           + 16;
}

void lbm_pull_tma_box(int dtype, int nx, int* bx, int* by, int* halo) {
    *bx = pull_bx(dtype, nx);
    *by = 256 / *bx;
    *halo = dtype == 0 ? 4 : 2;
}

// maps[0]: box (BX, BY, 1), maps[1]: box (BX + A, BY, 1) over the source lattice as (x, y, 19 nz)
cudaError_t lbm_pull_tma_launch(int dtype, bool exact, int mode, bool pdl, const CUtensorMap* maps, const void* src,
                                void* dst, const uint8_t* fl2, const LbmParams& p, int grid, int stages,
                                cudaStream_t s) {
    if (dtype == 1) return exact ? pull_t<double, true, 32>(mode, pdl, maps, src, dst, fl2, p, grid, stages, s)
                                 : pull_t<double, false, 32>(mode, pdl, maps, src, dst, fl2, p, grid, stages, s);
    if (pull_bx(dtype, p.nx) == 128)
        return exact ? pull_t<float, true, 128>(mode, pdl, maps, src, dst, fl2, p, grid, stages, s)
                     : pull_t<float, false, 128>(mode, pdl, maps, src, dst, fl2, p, grid, stages, s);
    return exact ? pull_t<float, true, 64>(mode, pdl, maps, src, dst, fl2, p, grid, stages, s)
                 : pull_t<float, false, 64>(mode, pdl, maps, src, dst, fl2, p, grid, stages, s);
}

}  // namespace st35d
