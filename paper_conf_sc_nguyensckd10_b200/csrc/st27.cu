// st27.cu — 3.5D-blocked sweep of the 27-point stencil (
// SURVEY §8(f) f1): B = alpha*C + beta*F + gamma*E + delta*K over the 3x3x3
// cube (centre, 6 faces, 12 edges, 8 corners), Jacobi two-grid sweeps,
// Dirichlet shell (X1), dim_T levels kept on chip.
// This kernel is the BIT-EXACT build (the oracle's X24 operation order); the
// tolerance build runs st27t_kernel.cuh on the 7-point machinery.
//
// Mapping (B200, sm_100a).  One CTA = a 32 x 32 loaded XY tile (8 warps of
// 32 lanes x 4 rows FP32, 32 x 16 with 2 rows FP64) streamed along a Z chunk,
// two CTAs per SM (<= 128 registers) so one CTA's barrier waits overlap the
// other's work (measured at 256^3 FP32 dim_T 2: 16 warps x 2 rows 329, x 4
// rows 351, 8 warps x 4 rows 408, x 8 rows 247 Gupd/s).  The 27-point sum factorises
// by plane (reading X24): for every plane of a level each point forms
//   v = a[y-1] + a[y+1],  h = a[x-1] + a[x+1],  f = h + v,  e = v[x-1] + v[x+1]
// once (x pairs by warp shuffle, the y neighbours of a warp's edge rows
// through a 4/8 KB shared-memory plane), and keeps (a, f, e) of the last three
// planes of every level in registers (the Z window; its slot rotation is a
// compile-time index in each of three round bodies, no moves).  A level-(t+1) point is then
//   F = f0 + (a- + a+),  E = e0 + (f- + f+),  K = e- + e+,
//   B = ((alpha*a0 + beta*F) + gamma*E) + delta*K
// — 12 adds + 4 products per point and level instead of the 26 + 4 the
// definition spells out, the same operation order as the oracle's
// (bit-identical with EXACT, tolerance with FMA contraction otherwise).
// Level t of round i is plane lo0 + i - t (lag 1 per level, P:251 with the
// levels run in order under a CTA barrier); every level runs every round so the
// windows stay aligned, results outside a level's valid region are never
// stored.  The valid region shrinks by one point per level on every tile side
// that is not the grid shell, so a tile stores its inner (32-2D)^2 points
// (P:216); the last tile in X and Y is shifted back inside the grid (X15) and
// Z chunks re-read D planes on each side (flexible balance).
#include <cstdio>
#include <type_traits>
#include "launch.h"

namespace st35d {

#ifndef ST27_STEP3
#define ST27_STEP3 0
#endif

namespace {
template <typename T, bool EX> struct Op;
template <> struct Op<float, true> {
    static __device__ __forceinline__ float add(float a, float b) { return __fadd_rn(a, b); }
    static __device__ __forceinline__ float mul(float a, float b) { return __fmul_rn(a, b); }
};
template <> struct Op<double, true> {
    static __device__ __forceinline__ double add(double a, double b) { return __dadd_rn(a, b); }
    static __device__ __forceinline__ double mul(double a, double b) { return __dmul_rn(a, b); }
};
template <typename T> struct Op<T, false> {
    static __device__ __forceinline__ T add(T a, T b) { return a + b; }
    static __device__ __forceinline__ T mul(T a, T b) { return a * b; }
};

constexpr int TW = 32;       // loaded tile width (one warp)
#ifndef ST27_NWARP
#define ST27_NWARP 8
#endif
constexpr int NWARP = ST27_NWARP;
constexpr int NTHR = TW * NWARP;
constexpr int MINB = 512 / NTHR;   // CTAs per SM at <= 128 registers
#ifndef ST27_VY32
#define ST27_VY32 4
#endif
// loaded tile height = NWARP x rows per thread: FP32 32 (4 per thread), FP64 16 (2)
#ifndef ST27_VY64
#define ST27_VY64 2
#endif
template <typename T> constexpr int vy_of() { return sizeof(T) == 4 ? ST27_VY32 : ST27_VY64; }
template <typename T> constexpr int th_of() { return NWARP * vy_of<T>(); }
}  // namespace

struct St27Params {
    int nx, ny, nz, ntx, nty, zchunk;
    double alpha, beta, gamma, delta;
};

template <typename T, int D, bool EX>
__global__ void __launch_bounds__(NTHR, MINB) st27_kernel(const T* __restrict__ a, T* __restrict__ b, St27Params p) {
    using O = Op<T, EX>;
    constexpr int VY = vy_of<T>(), TH = th_of<T>();
    __shared__ T sm[2][TH][TW];
    const int lane = threadIdx.x, w = threadIdx.y;
    const int tiles = p.ntx * p.nty;
    const int tile = blockIdx.x % tiles, zc = blockIdx.x / tiles;
    const int wx = TW - 2 * D, wy = TH - 2 * D;
    int x0 = (tile % p.ntx) * wx, y0 = (tile / p.ntx) * wy;
    x0 = max(0, min(x0, p.nx - TW));
    y0 = max(0, min(y0, p.ny - TH));
    const int gx = x0 + lane, cx = min(gx, p.nx - 1);
    const int zs = zc * p.zchunk, ze = min(p.nz, zs + p.zchunk);
    const int lo0 = max(0, zs - D), hi0 = min(p.nz, ze + D);
    const int nround = (hi0 - lo0) + D;
    const T alpha = T(p.alpha), beta = T(p.beta), gamma = T(p.gamma), delta = T(p.delta);
    const size_t plane = (size_t)p.nx * p.ny;

    int gy[VY];
    bool shxy[VY], st[VY];
    size_t off[VY];
    const bool xin = (x0 == 0 ? gx >= 0 : gx >= x0 + D) && (x0 + TW >= p.nx ? gx < p.nx : gx < x0 + TW - D);
#pragma unroll
    for (int j = 0; j < VY; ++j) {
        gy[j] = y0 + w * VY + j;
        const int cy = min(gy[j], p.ny - 1);
        off[j] = (size_t)cy * p.nx + cx;
        shxy[j] = gx == 0 || gx == p.nx - 1 || gy[j] == 0 || gy[j] == p.ny - 1;
        const bool yin = (y0 == 0 ? true : gy[j] >= y0 + D) && (y0 + TH >= p.ny ? gy[j] < p.ny : gy[j] < y0 + TH - D);
        st[j] = xin && yin;
    }

    // Z windows: level L (0..D-1) as a source, slot k holds (a, f, e) of one plane
    T wa[D][3][VY], wf[D][3][VY], we[D][3][VY];
    // zero-initialised: the first rounds of a chunk read window slots that no
    // earlier round has written (their results are never stored, but reading
    // an indeterminate value is undefined behaviour the compiler may exploit)
#pragma unroll
    for (int L = 0; L < D; ++L)
#pragma unroll
        for (int k = 0; k < 3; ++k)
#pragma unroll
            for (int j = 0; j < VY; ++j) wa[L][k][j] = wf[L][k][j] = we[L][k][j] = T(0);
    // level-0 planes arrive PF-1 rounds ahead through a per-thread cp.async
    // ring (each thread copies and later reads only its own VY elements, so no
    // barrier guards the ring; the loads stay in flight across the rounds'
    // barriers instead of stalling every round on HBM latency)
#ifndef ST27_PF
#define ST27_PF 3
#endif
    constexpr int PF = ST27_PF;
    __shared__ T ring[PF][TH][TW];
    const T* gnext = a + (size_t)lo0 * plane;                  // next level-0 plane to copy
    int pnext = lo0;
    uint32_t off32[VY];
#pragma unroll
    for (int j = 0; j < VY; ++j) off32[j] = (uint32_t)off[j];
    const uint32_t ring0 = smem_u32(&ring[0][w * VY][lane]);
    auto issue = [&](int slot) {
#pragma unroll
        for (int j = 0; j < VY; ++j)
            asm volatile("cp.async.ca.shared.global [%0], [%1], %2;"
                         ::"r"(ring0 + (uint32_t)((slot * TH + j) * TW * sizeof(T))), "l"(gnext + off32[j]),
                         "n"(sizeof(T)) : "memory");
        asm volatile("cp.async.commit_group;" ::: "memory");
        if (pnext < hi0 - 1) { gnext += plane; ++pnext; }    // past the chunk: re-copy the last plane
    };
#pragma unroll
    for (int k = 0; k < PF - 1; ++k) issue(k);
    int rslot = 0;                                             // ring slot of this round's plane
    int buf = 0;

    // one round with compile-time window rotation R: slot (R+2)%3 receives the
    // new plane, (R+1)%3 holds the middle, R%3 the lowest
    auto round = [&](int i, auto Rc, auto Sc) {
        constexpr int R = decltype(Rc)::value;
        constexpr bool SHELL = decltype(Sc)::value;           // false: no shell point in this round
        constexpr int sN = (R + 2) % 3, sC = (R + 1) % 3, sM = R % 3;
        T v[VY];
        issue(rslot == 0 ? PF - 1 : rslot - 1);                // slot of plane i-1, already read
        asm volatile("cp.async.wait_group %0;" ::"n"(PF - 1) : "memory");
#pragma unroll
        for (int j = 0; j < VY; ++j) v[j] = ring[rslot][w * VY + j][lane];
        rslot = rslot == PF - 1 ? 0 : rslot + 1;
#pragma unroll
        for (int L = 0; L <= D; ++L) {
            const int q = lo0 + i - L;                          // plane of level L this round
            if (L > 0) {                                        // level L from the window of level L-1
                const bool shz = q == 0 || q == p.nz - 1;
#pragma unroll
                for (int j = 0; j < VY; ++j) {
                    const T c0 = wa[L - 1][sC][j];
                    const T zs2 = O::add(wa[L - 1][sM][j], wa[L - 1][sN][j]);
                    const T F = O::add(wf[L - 1][sC][j], zs2);
                    const T E = O::add(we[L - 1][sC][j], O::add(wf[L - 1][sM][j], wf[L - 1][sN][j]));
                    const T K = O::add(we[L - 1][sM][j], we[L - 1][sN][j]);
                    const T r = O::add(O::add(O::add(O::mul(alpha, c0), O::mul(beta, F)), O::mul(gamma, E)),
                                       O::mul(delta, K));
                    if constexpr (SHELL) v[j] = (shxy[j] || shz) ? c0 : r;
                    else v[j] = r;
                }
            }
            if (L == D) {                                       // final level: store the tile interior
                if (q >= zs && q < ze) {
                    T* ob = b + (size_t)q * plane;
#pragma unroll
                    for (int j = 0; j < VY; ++j)
                        if (st[j]) ob[off32[j]] = v[j];
                }
                break;
            }
            // in-plane partial sums of level L, plane q
            sm[buf][w * VY][lane] = v[0];
            sm[buf][w * VY + VY - 1][lane] = v[VY - 1];
            __syncthreads();
            const T up = sm[buf][max(w * VY - 1, 0)][lane];
            const T dn = sm[buf][min(w * VY + VY, TH - 1)][lane];
            buf ^= 1;
#pragma unroll
            for (int j = 0; j < VY; ++j) {
                const T ym = j == 0 ? up : v[j - 1];
                const T yp = j == VY - 1 ? dn : v[j + 1];
                const T vv = O::add(ym, yp);
                const T xm = __shfl_up_sync(0xffffffffu, v[j], 1), xp = __shfl_down_sync(0xffffffffu, v[j], 1);
                const T f = O::add(O::add(xm, xp), vv);
                const T vm = __shfl_up_sync(0xffffffffu, vv, 1), vp = __shfl_down_sync(0xffffffffu, vv, 1);
                wa[L][sN][j] = v[j];
                wf[L][sN][j] = f;
                we[L][sN][j] = O::add(vm, vp);
            }
        }
    };
    // rotation chosen per round: the same three bodies called in sequence
    // from a loop stepping by three rounds gave wrong values from the fourth
    // round on (cause not isolated)
    // (CTA-uniform) rounds of tiles off the XY shell whose levels' planes miss
    // z = 0 and z = nz-1 take a body without the per-point shell select
    const bool tile_shell = x0 == 0 || x0 + TW >= p.nx || y0 == 0 || y0 + TH >= p.ny;
    using S1 = std::true_type;
    using S0 = std::false_type;
#if ST27_STEP3
    // A/B: the three rotation bodies in sequence from a loop stepping by three
    for (int i = 0; i < nround; i += 3) {
        const bool sh0 = tile_shell || lo0 + i - D <= 0 || lo0 + i - 1 >= p.nz - 1;
        if (sh0) round(i, std::integral_constant<int, 0>{}, S1{}); else round(i, std::integral_constant<int, 0>{}, S0{});
        if (i + 1 >= nround) break;
        const bool sh1 = tile_shell || lo0 + i + 1 - D <= 0 || lo0 + i >= p.nz - 1;
        if (sh1) round(i + 1, std::integral_constant<int, 1>{}, S1{}); else round(i + 1, std::integral_constant<int, 1>{}, S0{});
        if (i + 2 >= nround) break;
        const bool sh2 = tile_shell || lo0 + i + 2 - D <= 0 || lo0 + i + 1 >= p.nz - 1;
        if (sh2) round(i + 2, std::integral_constant<int, 2>{}, S1{}); else round(i + 2, std::integral_constant<int, 2>{}, S0{});
    }
#else
    for (int i = 0; i < nround; ++i) {
        const int r = i % 3;
        const bool sh = tile_shell || lo0 + i - D <= 0 || lo0 + i - 1 >= p.nz - 1;
        if (sh) {
            if (r == 0) round(i, std::integral_constant<int, 0>{}, S1{});
            else if (r == 1) round(i, std::integral_constant<int, 1>{}, S1{});
            else round(i, std::integral_constant<int, 2>{}, S1{});
        } else {
            if (r == 0) round(i, std::integral_constant<int, 0>{}, S0{});
            else if (r == 1) round(i, std::integral_constant<int, 1>{}, S0{});
            else round(i, std::integral_constant<int, 2>{}, S0{});
        }
    }
#endif
    // the last rounds re-copy the chunk's last plane into the ring: drain them
    asm volatile("cp.async.wait_all;" ::: "memory");
}

template <typename T, int D, bool EX>
static cudaError_t launch_one(const void* in, void* out, St27Params p, int sms, cudaStream_t s, int* grid_out);

// Z chunking: the CTAs of one depth-D sweep are ntiles x nchunks; pick the
// chunk count that minimises (waves) x (rounds per chunk), each chunk paying
// its 2D re-read planes and D drain rounds (flexible balance).
static int choose_chunks(int ntiles, int nz, int D, int slots);

template <typename T, int D, bool EX>
static cudaError_t launch_one(const void* in, void* out, St27Params p, int sms, cudaStream_t s, int* grid_out) {
    static int occ = 0;
    if (!occ && cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, st27_kernel<T, D, EX>, NTHR, 0) != cudaSuccess)
        return cudaGetLastError();
    const int ntiles = p.ntx * p.nty;
    p.zchunk = choose_chunks(ntiles, p.nz, D, sms * (occ > 0 ? occ : 1));
    const int grid = ntiles * ((p.nz + p.zchunk - 1) / p.zchunk);
    if (grid_out) *grid_out = grid;
    st27_kernel<T, D, EX><<<grid, dim3(TW, NWARP), 0, s>>>(static_cast<const T*>(in), static_cast<T*>(out), p);
    return cudaGetLastError();
}

template <typename T, bool EX>
static cudaError_t dispatch(int D, const void* in, void* out, const St27Params& p, int sms, cudaStream_t s,
                            int* grid_out) {
    switch (D) {
        case 1: return launch_one<T, 1, EX>(in, out, p, sms, s, grid_out);
        case 2: return launch_one<T, 2, EX>(in, out, p, sms, s, grid_out);
        case 3: if constexpr (sizeof(T) == 4) return launch_one<T, 3, EX>(in, out, p, sms, s, grid_out); else break;
        case 4: if constexpr (sizeof(T) == 4) return launch_one<T, 4, EX>(in, out, p, sms, s, grid_out); else break;
        default: break;
    }
    return cudaErrorInvalidValue;
}

static int choose_chunks(int ntiles, int nz, int D, int slots) {
    int best = 1;
    double bestc = 1e300;
    for (int nch = 1; nch <= nz; ++nch) {
        const int zch = (nz + nch - 1) / nch;
        if (zch < 2 && nch > 1) break;
        const int ctas = ntiles * ((nz + zch - 1) / zch);
        const double waves = (double)((ctas + slots - 1) / slots);
        const double cost = waves * (zch + 3.0 * D);
        if (cost < bestc - 1e-9) { bestc = cost; best = nch; }
    }
    return (nz + best - 1) / best;
}

// FP64 at D >= 3 spills under the 128-register cap (FP32 D = 4 spills too, kept for the sweep)
int st27_depth_max(int dtype) { return dtype == 0 ? 4 : 2; }

cudaError_t st27_launch(int dtype, bool exact, int D, const void* in, void* out, int nx, int ny, int nz, double alpha,
                        double beta, double gamma, double delta, int sms, cudaStream_t s, int* grid_out) {
    if (D < 1 || D > st27_depth_max(dtype)) return cudaErrorInvalidValue;
    if ((size_t)nx * ny >= (size_t(1) << 32)) return cudaErrorInvalidValue;   // 32-bit in-plane offsets
    St27Params p;
    p.nx = nx; p.ny = ny; p.nz = nz;
    p.ntx = nx <= TW ? 1 : 1 + (nx - TW + (TW - 2 * D) - 1) / (TW - 2 * D);
    const int TH = dtype == 0 ? th_of<float>() : th_of<double>();
    p.nty = ny <= TH ? 1 : 1 + (ny - TH + (TH - 2 * D) - 1) / (TH - 2 * D);
    p.zchunk = 0;
    if (dtype == 0) { p.alpha = (float)alpha; p.beta = (float)beta; p.gamma = (float)gamma; p.delta = (float)delta; }
    else { p.alpha = alpha; p.beta = beta; p.gamma = gamma; p.delta = delta; }
    // the tolerance build runs st27t_kernel.cuh (7-point machinery); this kernel is the bit-exact one
    if (!exact) return cudaErrorInvalidValue;
    return dtype == 0 ? dispatch<float, true>(D, in, out, p, sms, s, grid_out)
                      : dispatch<double, true>(D, in, out, p, sms, s, grid_out);
}

}  // namespace st35d
