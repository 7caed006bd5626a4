// api.cu — the C ABI (include/st35d.h): plan, planner, sweep driver,
// TMA descriptors, host-pointer staging.  No torch types cross this boundary.
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <string>
#include <vector>
#include <algorithm>
#include <cudaTypedefs.h>
#include <dlfcn.h>
#include <nvtx3/nvToolsExt.h>

#include "../../include/st35d.h"
#include "launch.h"
#include "dist.h"
#include "st13_kernel.cuh"
#include "st27t_kernel.cuh"

using namespace st35d;

// NCCL CTAs per communicator (ncclConfig_t.maxCTAs): the ghost exchange is a few
// MB per sweep, a handful of CTAs saturate NVLink for it, the rest stay with the sweep
constexpr int ST_NCCL_MAX_CTAS = 4;

// NVTX3 ranges (header-only; no cost without an attached tool): one per C-ABI
// run and one per sweep / pass / ghost exchange, for nsys / ncu range filters
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange&) = delete;
    NvtxRange& operator=(const NvtxRange&) = delete;
};

// ----------------------------------------------------------------------------
// errors
// ----------------------------------------------------------------------------
static thread_local std::string g_err;
static thread_local int g_code = 0;

static int fail(int code, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    g_code = code;
    return code;
}
#define CUDA_TRY(x)                                                                          \
    do {                                                                                     \
        cudaError_t e_ = (x);                                                                \
        if (e_ != cudaSuccess) return fail(ST_ECUDA, "%s: %s (%s:%d)", #x, cudaGetErrorString(e_), __FILE__, __LINE__); \
    } while (0)

extern "C" const char* st_last_error(void) { return g_err.c_str(); }
extern "C" int st_last_status(void) { return g_code; }

// ----------------------------------------------------------------------------
// TMA descriptor encoding through the driver entry point (no -lcuda needed)
// ----------------------------------------------------------------------------
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    if (!fn) {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    }
    return fn;
}

static int encode_3d(CUtensorMap* map, const void* base, st_dtype dt, int nx, int ny, int nz, int bx, int by) {
    auto enc = get_encode();
    if (!enc) return fail(ST_ECUDA, "cuTensorMapEncodeTiled unavailable");
    const size_t E = dt == ST_F32 ? 4 : 8;
    cuuint64_t dims[3] = {(cuuint64_t)nx, (cuuint64_t)ny, (cuuint64_t)nz};
    cuuint64_t strides[2] = {(cuuint64_t)nx * E, (cuuint64_t)nx * ny * E};
    cuuint32_t box[3] = {(cuuint32_t)bx, (cuuint32_t)by, 1};
    cuuint32_t es[3] = {1, 1, 1};
    // L2 promotion: the tile boxes start at arbitrary 16-byte offsets, so a
    // 256-byte promotion would fetch up to twice the requested sectors
    CUtensorMapL2promotion promo = CU_TENSOR_MAP_L2_PROMOTION_NONE;
    CUresult r = enc(map, dt == ST_F32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3,
                     const_cast<void*>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, promo, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return fail(ST_ECUDA, "cuTensorMapEncodeTiled failed (%d) box %dx%d", (int)r, bx, by);
    return ST_OK;
}

// SoA D3Q19 lattice as one 3D map (x, y, 19 nz): population i is planes [i nz, i nz + nz)
static int encode_lbm(CUtensorMap* map, const void* base, st_dtype dt, int nx, int ny, int nz, int bx, int by) {
    if (19LL * nz > (1LL << 31) - 1) return fail(ST_EUNSUPPORTED, "19 nz exceeds a TMA coordinate");
    return encode_3d(map, base, dt, nx, ny, 19 * nz, bx, by);
}

// ----------------------------------------------------------------------------
// plan
// ----------------------------------------------------------------------------
struct Geo7 {
    int d = 0, VY = 0, NTX = 0, VX = 0, TX = 0, NTY = 0, TY = 0;
    int hx = 0, wx = 0, wy = 0, tiles_x = 0, tiles_y = 0, threads = 0, grid = 0, ring = 0;
    int ey = 0, ly_last = 0, oy0_last = 0;   // y placement (St7Params)
    int maxt = 0;                            // threads of the kernel variant (>= threads launched)
    int minb = 1;                            // CTAs per SM of the variant
    int vxk = 0;                             // points per thread row (0: the dtype's 16-byte vector)
    size_t smem = 0;
    double kappa = 0;
    St7LaunchFn fn = nullptr;
    St13LaunchFn fn13 = nullptr;             // radius-2 plans
    St27tLaunchFn fn27t = nullptr;           // 27-point plans (tolerance build)
};

struct st_plan {
    int nx, ny, nz;
    st_dtype dtype;
    int dimT;
    int dimK = 0;      // sweep depth of st7_run (<= dimT; st_plan_autotune may lower it)
    int dimKmax = 0;   // deepest sweep the 7-point kernels can tile (<= dimT)
    int dev = 0, sms = 0;
    size_t smem_optin = 0;
    size_t smem_sm = 0;        // shared memory per SM
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    bool exact = false;
    int variant = ST_VARIANT_35D;    // st_plan_set_variant (ablation baseline ST_VARIANT_NAIVE)
    double lid[3] = {0.05, 0.0, 0.0};
    int launches = 0;
    // st_plan_set_option (include/st35d.h): tuning / test selections, no environment variables
    int opt_lbm_batched = -1;   // -1 auto
    int opt_lbm_kernel = 0;     // 0 auto, 1 push, 2 multi-level, 3 gather form, 4 gather form + TMA pulls
    int opt_lbm_stages = 0;     // TMA pull ring depth (0 auto)
    int last_lbm_kernel = 0;    // kernel code of the last lbm_d3q19_run (st_plan_get_info)
    int opt_overlap = 1;
    int opt_pdl = 1;
    int opt_st7_variant = 0;    // 0 auto, else VY * 1000 + threads per CTA (+ 10000 * CTAs per SM)
    int opt_zchunk = 0;         // 0: z-runs as the work split gives; > 0: 3D blocks of that depth
    // host-pointer staging
    void* hbuf[2] = {nullptr, nullptr};
    size_t hbuf_bytes = 0;
    uint8_t* hflags = nullptr;
    size_t hflags_bytes = 0;
    int* d_count = nullptr;
    int* h_count = nullptr;
    const void* flags_checked = nullptr;
    uint8_t* fl2 = nullptr;          // flags | 0x80 (FLUID next to non-FLUID), lbm_35d input
    size_t fl2_bytes = 0;
    // distribution (Z slabs)
    Dist dist;
    std::map<int, Geo7> geo7;  // by depth
};

static size_t esize(st_dtype d) { return d == ST_F32 ? 4 : 8; }
struct GeoL { int TY = 0, wx = 0, wy = 0, tiles_x = 0, tiles_y = 0; size_t smem = 0; };
static int planL(const st_plan* p, int d, GeoL& g);
static int max_lbm_depth(const st_plan* p);
static bool lbm_use_push(const st_plan* p);

// Kernel variant (rows per thread VY, threads per CTA) for a sweep depth.
// Registers (ptxas -v) cap what fits: VY = 4 keeps 2 planes x 16 points per
// level in registers and fits 256 threads up to dim_T = 4 without spills;
// deeper sweeps use VY = 2 (half the window per thread, twice the exchange
// traffic per point).  ST_OPT_ST7_VARIANT overrides (A/B).
static void variant_for(const st_plan* p, int d, int& vy, int& nt, int& minb, int& vx) {
    minb = 1;
    vx = 0;
    if (p->opt_st7_variant) {
        const int v = p->opt_st7_variant;
        vy = v / 1000 % 10; nt = v % 1000; minb = std::max(1, v / 10000 % 10); vx = v / 100000;
        return;
    }
    vy = d <= 4 ? 4 : 2;
    nt = 256;
    // FP32 dim_T <= 4 on grids with long z-runs per CTA (~64x60 tiles x planes over
    // the SMs): the narrow layout (2 points per thread row, no constructed pairs)
    // with 16 warps per SM; measured on B200 512^3 dim_T 4: 1600 vs 1385 Gupd/s,
    // while 256^3 (43 planes per CTA, restart-bound) prefers 8 wide warps (1239 vs 1171)
    const double run = (double)p->nx * p->ny / (64.0 * 60.0) * p->dist.nzl / std::max(1, p->sms);
    if (p->dtype == ST_F32 && d <= 4 && run >= 150.0) { vx = 2; nt = 512; return; }
    // FP64 (2 doubles per 16-byte vector, 32 threads per tile row): VY = 2 gives
    // 16-row tiles, too short for dim_T >= 7 (written rows 16 - 2 dim_T)
    if (p->dtype == ST_F64) vy = (d <= 4 || d >= 7) ? 4 : 2;   // measured 256^3 dim_T 4: VY 4 699, VY 2 385 Gupd/s
}

static St7LaunchFn lookup7(st_dtype dt, bool exact, int d, int vy, int nt, int minb, int vx = 0) {
    if (dt == ST_F32) return exact ? st7_lookup_f32_exact(d, vy, nt, minb, vx) : st7_lookup_f32_fast(d, vy, nt, minb, vx);
    return exact ? st7_lookup_f64_exact(d, vy, nt, minb, vx) : st7_lookup_f64_fast(d, vy, nt, minb, vx);
}

// CTAs per SM of a variant (minb 9 = the ladder's level-by-level kernel, one per SM)
static int ctas_per_sm(const Geo7& g) { return g.minb == 9 ? 1 : g.minb; }

static size_t smem7(const Geo7& g, st_dtype dt, int ring) {
    // TMA ring + row exchange [D-1][2][2][threads] x one thread row (VX points: 16 B, or
    // 8 B for the narrow FP32 layout) + mbarriers
    return (size_t)ring * g.TX * g.TY * esize(dt) +
           (size_t)(g.d > 1 ? g.d - 1 : 0) * 4 * g.threads * (g.VX * esize(dt)) + ST7_RING_MAX * 8;
}

// Planner for one sweep depth d over an nx x ny plane with nzo output planes:
// eq. (1) analog (on-chip bytes of one SM: register file for the Z window,
// shared memory for the TMA ring and the Y exchange), then the XY tile that
// minimises computed points per plane (halo + ragged last tile), then a
// persistent grid of one CTA per SM with equal (tile, z) volume per CTA.
// y placement of a tile height (see st7_tile in st7_kernel.cuh): the regular
// tiles are shifted down by ey so that y = 0 is the last row of a thread's
// block, the last tile is placed so that y = ny-1 is the first row of a block;
// no halo is needed beyond a grid face (the shell is fixed), so the first and
// last tiles write up to the face
// (R = stencil radius: the shell is R rows thick and the halo R*d rows)
static void place_y(Geo7& g, int ny, int d, int R = 1) {
    const int h = R * d;
    g.wy = g.TY - 2 * h;
    g.ey = ((g.VY - R - h) % g.VY + g.VY) % g.VY;   // y = R-1 on the last row of a block
    g.ly_last = g.oy0_last = 0;
    if (g.TY - h - g.ey >= ny) { g.tiles_y = 1; return; }
    g.ly_last = ny - R - (g.TY - g.VY);              // y = ny-R on the first row of a block
    g.oy0_last = std::max(g.ly_last + h, 0);
    g.tiles_y = std::max(1, (g.oy0_last + g.ey + g.wy - 1) / g.wy) + 1;
}

static int plan7(st_plan* p, int d, int nzo, Geo7& g) {
    g.d = d;
    int ntmax = 0, vx = 0;
    variant_for(p, d, g.VY, ntmax, g.minb, vx);
    g.vxk = vx;
    g.VX = vx ? vx : (p->dtype == ST_F32 ? 4 : 2);
    g.NTX = 64 / g.VX;
    g.TX = g.NTX * g.VX;
    // TMA boxes must start on a 16-byte boundary: halo and written width in
    // 16-byte units (4 FP32 / 2 FP64 points) whatever the points per thread
    const int al16 = (int)(16 / esize(p->dtype));
    g.hx = (d + al16 - 1) / al16 * al16;
    g.wx = (g.TX - g.hx - d) & ~(al16 - 1);
    if (g.wx < g.VX) return fail(ST_EUNSUPPORTED, "dim_T %d too deep for the %d-wide tile of this build", d, g.TX);
    g.tiles_x = (p->nx + g.wx - 1) / g.wx;
    // tile height: the thread-row count (<= the variant's threads) that loads
    // the fewest rows per plane (tiles_y * TY); ties go to the taller tile
    long best = -1;
    for (int nty = 2; nty <= ntmax / g.NTX; ++nty) {
        Geo7 c = g;
        c.NTY = nty;
        c.TY = nty * c.VY;
        c.threads = c.NTX * nty;
        if (c.TY - 2 * d < 1) continue;
        place_y(c, p->ny, d);
        // TMA ring: as deep as shared memory allows (the loads run ring-2 planes
        // ahead and must cover HBM latency, several rounds of compute)
        c.ring = 0;
        for (int r = ST7_RING_MAX; r >= 4; --r)
            if (smem7(c, p->dtype, r) <= (ctas_per_sm(g) == 1 ? p->smem_optin : p->smem_sm / ctas_per_sm(g) - 1024)) {
                c.ring = r;
                break;
            }
        if (c.ring < 4) continue;
        c.smem = smem7(c, p->dtype, c.ring);
        const long cost = (long)c.tiles_y * c.TY;
        if (best < 0 || cost < best || (cost == best && c.TY > g.TY)) { best = cost; g = c; }
    }
    if (best < 0) return fail(ST_EUNSUPPORTED, "dim_T %d too deep for the tiles of this build", d);
    const long long work = (long long)g.tiles_x * g.tiles_y * nzo;
    g.grid = (int)std::min<long long>((long long)p->sms * ctas_per_sm(g), std::max<long long>(work, 1));
    g.kappa = (double)g.tiles_x * g.TX * g.tiles_y * g.TY / ((double)p->nx * p->ny);
    g.fn = lookup7(p->dtype, p->exact, d, g.VY, ntmax, g.minb, g.vxk);
    if (!g.fn) return fail(ST_EUNSUPPORTED, "no kernel for dim_T %d (VY %d, %d threads)", d, g.VY, ntmax);
    g.maxt = ntmax;
    return ST_OK;
}

static int get_geo7(st_plan* p, int d, int nzo, Geo7*& out) {
    auto it = p->geo7.find(d);
    if (it == p->geo7.end() ||
        it->second.fn != lookup7(p->dtype, p->exact, d, it->second.VY, it->second.maxt, it->second.minb, it->second.vxk)) {
        Geo7 g;
        int rc = plan7(p, d, nzo, g);
        if (rc) return rc;
        it = p->geo7.insert_or_assign(d, g).first;
    }
    out = &it->second;
    // grid depends on the output-plane count of the call
    const long long work = (long long)out->tiles_x * out->tiles_y * nzo;
    out->grid = (int)std::min<long long>((long long)p->sms * ctas_per_sm(*out), std::max<long long>(work, 1));
    return ST_OK;
}


// ----------------------------------------------------------------------------
// radius-2 (13-point star) planner: the 7-point planner with R = 2 (halo 2d,
// shell 2 rows thick, ring keeps 3 planes, exchange 2 rows per side for 3 rounds)
// ----------------------------------------------------------------------------
static size_t smem13(const Geo7& g, st_dtype dt, int ring) {
    return (size_t)ring * g.TX * g.TY * esize(dt) + (size_t)(g.d > 1 ? g.d - 1 : 0) * 3 * 4 * g.threads * 16 +
           ST7_RING_MAX * 8;
}

static int plan13(st_plan* p, int d, int nzo, Geo7& g) {
    const int R = 2;
    g.d = d;
    g.VX = p->dtype == ST_F32 ? 4 : 2;
    g.NTX = p->dtype == ST_F32 ? 16 : 32;
    g.TX = g.NTX * g.VX;
    g.VY = d <= 2 ? 4 : 2;
    g.maxt = 256;
    g.minb = 1;
    g.hx = (R * d + g.VX - 1) / g.VX * g.VX;
    g.wx = (g.TX - g.hx - R * d) & ~(g.VX - 1);
    if (g.wx < g.VX) return fail(ST_EUNSUPPORTED, "radius 2: dim_T %d too deep for the %d-wide tile", d, g.TX);
    g.tiles_x = (p->nx + g.wx - 1) / g.wx;
    long best = -1;
    for (int nty = 2; nty <= g.maxt / g.NTX; ++nty) {
        Geo7 c = g;
        c.NTY = nty;
        c.TY = nty * c.VY;
        c.threads = c.NTX * nty;
        if (c.TY - 2 * R * d < 1) continue;
        place_y(c, p->ny, d, R);
        c.ring = 0;
        for (int r = ST7_RING_MAX; r >= 4; --r)
            if (smem13(c, p->dtype, r) <= p->smem_optin) { c.ring = r; break; }
        if (c.ring < 4) continue;
        c.smem = smem13(c, p->dtype, c.ring);
        const long cost = (long)c.tiles_y * c.TY;
        if (best < 0 || cost < best || (cost == best && c.TY > g.TY)) { best = cost; g = c; }
    }
    if (best < 0) return fail(ST_EUNSUPPORTED, "radius 2: dim_T %d too deep for the tiles of this build", d);
    const long long work = (long long)g.tiles_x * g.tiles_y * nzo;
    g.grid = (int)std::min<long long>(p->sms, std::max<long long>(work, 1));
    g.kappa = (double)g.tiles_x * g.TX * g.tiles_y * g.TY / ((double)p->nx * p->ny);
    g.fn13 = st13_lookup(p->dtype == ST_F32 ? 0 : 1, p->exact, d, g.VY);
    if (!g.fn13) return fail(ST_EUNSUPPORTED, "no radius-2 kernel for dim_T %d", d);
    return ST_OK;
}

// ----------------------------------------------------------------------------
// 27-point planner (st27t_kernel.cuh, tolerance build): the 7-point planner with
// R = 1 and the exchange double-buffered by round parity; VY = 4 rows per thread
// up to depth vy4_max, else 2
// ----------------------------------------------------------------------------
static size_t smem27t(const Geo7& g, st_dtype dt, int ring) {
    return (size_t)ring * g.TX * g.TY * esize(dt) + (size_t)(g.d > 1 ? g.d - 1 : 0) * 4 * g.threads * 16 +
           ST7_RING_MAX * 8;
}

static int plan27t(st_plan* p, int d, int nzo, Geo7& g) {
    g.d = d;
    g.VX = p->dtype == ST_F32 ? 4 : 2;
    g.NTX = p->dtype == ST_F32 ? 16 : 32;
    g.TX = g.NTX * g.VX;
    g.VY = d <= ST27T_VY4_MAX ? 4 : 2;
    g.maxt = 256;
    g.minb = 1;
    g.hx = (d + g.VX - 1) / g.VX * g.VX;
    g.wx = (g.TX - g.hx - d) & ~(g.VX - 1);
    if (g.wx < g.VX) return fail(ST_EUNSUPPORTED, "27-point: dim_T %d too deep for the %d-wide tile", d, g.TX);
    g.tiles_x = (p->nx + g.wx - 1) / g.wx;
    long best = -1;
    for (int nty = 2; nty <= g.maxt / g.NTX; ++nty) {
        Geo7 c = g;
        c.NTY = nty;
        c.TY = nty * c.VY;
        c.threads = c.NTX * nty;
        if (c.TY - 2 * d < 1) continue;
        place_y(c, p->ny, d, 1);
        c.ring = 0;
        for (int r = ST7_RING_MAX; r >= 4; --r)
            if (smem27t(c, p->dtype, r) <= p->smem_optin) { c.ring = r; break; }
        if (c.ring < 4) continue;
        c.smem = smem27t(c, p->dtype, c.ring);
        const long cost = (long)c.tiles_y * c.TY;
        if (best < 0 || cost < best || (cost == best && c.TY > g.TY)) { best = cost; g = c; }
    }
    if (best < 0) return fail(ST_EUNSUPPORTED, "27-point: dim_T %d too deep for the tiles of this build", d);
    const long long work = (long long)g.tiles_x * g.tiles_y * nzo;
    g.grid = (int)std::min<long long>(p->sms, std::max<long long>(work, 1));
    g.kappa = (double)g.tiles_x * g.TX * g.tiles_y * g.TY / ((double)p->nx * p->ny);
    g.fn27t = st27t_lookup(p->dtype == ST_F32 ? 0 : 1, d, g.VY);
    if (!g.fn27t) return fail(ST_EUNSUPPORTED, "no 27-point kernel for dim_T %d", d);
    return ST_OK;
}

extern "C" st_plan* st_plan_create(int nx, int ny, int nz, st_dtype dtype, int dim_T) {
    if (nx < 3 || ny < 3 || nz < 3) { fail(ST_EINVAL, "grid %dx%dx%d: every extent must be >= 3", nx, ny, nz); return nullptr; }
    if (dtype != ST_F32 && dtype != ST_F64) { fail(ST_EINVAL, "dtype %d", (int)dtype); return nullptr; }
    if (dim_T < 1 || dim_T > ST_MAX_DIM_T) { fail(ST_EINVAL, "dim_T %d not in [1, %d]", dim_T, ST_MAX_DIM_T); return nullptr; }
    if (((size_t)nx * esize(dtype)) % 16 != 0) {
        fail(ST_EUNSUPPORTED, "nx*sizeof(dtype) = %zu is not a multiple of 16 bytes (TMA row pitch)",
             (size_t)nx * esize(dtype));
        return nullptr;
    }
    int dev = 0, cnt = 0;
    if (cudaGetDeviceCount(&cnt) != cudaSuccess || cnt == 0) { fail(ST_ECUDA, "no CUDA device"); cudaGetLastError(); return nullptr; }
    cudaGetDevice(&dev);
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, dev) != cudaSuccess) { fail(ST_ECUDA, "cudaGetDeviceProperties"); return nullptr; }
    if (prop.major < 10) { fail(ST_EUNSUPPORTED, "needs sm_100a (found sm_%d%d)", prop.major, prop.minor); return nullptr; }
    st_plan* p = new st_plan();
    p->nx = nx; p->ny = ny; p->nz = nz; p->dtype = dtype; p->dimT = dim_T;
    p->dev = dev;
    p->sms = prop.multiProcessorCount;
    p->smem_optin = prop.sharedMemPerBlockOptin;
    p->smem_sm = prop.sharedMemPerMultiprocessor;
    if (cudaStreamCreateWithFlags(&p->stream, cudaStreamNonBlocking) != cudaSuccess) {
        fail(ST_ECUDA, "stream create"); delete p; return nullptr;
    }
    p->own_stream = true;
    if (cudaMalloc(&p->d_count, sizeof(int)) != cudaSuccess || cudaMallocHost(&p->h_count, sizeof(int)) != cudaSuccess) {
        fail(ST_ENOMEM, "scratch"); st_destroy(p); return nullptr;
    }
    p->dist.init_single(nz);
    // the 7-point sweep of depth dim_T must tile (D > D_max is an
    // error, not a silent shallower sweep)
    Geo7* g = nullptr;
    if (get_geo7(p, dim_T, nz, g) != ST_OK) {
        const std::string msg = g_err;
        const int code = g_code;
        st_destroy(p);
        fail(code, "%s", msg.c_str());
        return nullptr;
    }
    p->dimK = p->dimKmax = dim_T;
    g_err.clear();
    g_code = 0;
    return p;
}

extern "C" void st_destroy(st_plan* p) {
    if (!p) return;
    if (p->stream) cudaStreamSynchronize(p->stream);
    p->dist.destroy();
    for (void* b : p->hbuf) if (b) cudaFree(b);
    if (p->hflags) cudaFree(p->hflags);
    if (p->fl2) cudaFree(p->fl2);
    if (p->d_count) cudaFree(p->d_count);
    if (p->h_count) cudaFreeHost(p->h_count);
    if (p->own_stream && p->stream) cudaStreamDestroy(p->stream);
    delete p;
}

extern "C" int st_plan_set_stream(st_plan* p, void* s) {
    if (!p) return fail(ST_EINVAL, "NULL plan");
    if (p->own_stream && p->stream) { cudaStreamSynchronize(p->stream); cudaStreamDestroy(p->stream); }
    p->stream = static_cast<cudaStream_t>(s);
    p->own_stream = false;
    return ST_OK;
}

extern "C" int st_plan_set_lbm_lid(st_plan* p, double ux, double uy, double uz) {
    if (!p) return fail(ST_EINVAL, "NULL plan");
    p->lid[0] = ux; p->lid[1] = uy; p->lid[2] = uz;
    return ST_OK;
}

extern "C" int st_plan_set_variant(st_plan* p, int variant) {
    if (!p) return fail(ST_EINVAL, "NULL plan");
    if (variant != ST_VARIANT_35D && variant != ST_VARIANT_NAIVE) return fail(ST_EINVAL, "variant %d", variant);
    p->variant = variant;
    return ST_OK;
}

extern "C" int st_plan_set_option(st_plan* p, int option, int value) {
    if (!p) return fail(ST_EINVAL, "NULL plan");
    switch (option) {
        case ST_OPT_LBM_BATCHED:
            if (value < -1 || value > 1) return fail(ST_EINVAL, "ST_OPT_LBM_BATCHED %d", value);
            p->opt_lbm_batched = value; return ST_OK;
        case ST_OPT_LBM_KERNEL:
            if (value < 0 || value > 4) return fail(ST_EINVAL, "ST_OPT_LBM_KERNEL %d", value);
            p->opt_lbm_kernel = value; return ST_OK;
        case ST_OPT_LBM_STAGES:
            if (value < 0 || value > 8) return fail(ST_EINVAL, "ST_OPT_LBM_STAGES %d", value);
            p->opt_lbm_stages = value; return ST_OK;
        case ST_OPT_OVERLAP: p->opt_overlap = value != 0; return ST_OK;
        case ST_OPT_PDL: p->opt_pdl = value != 0; return ST_OK;
        case ST_OPT_ZCHUNK:
            if (value < 0) return fail(ST_EINVAL, "ST_OPT_ZCHUNK %d", value);
            p->opt_zchunk = value;
            return ST_OK;
        case ST_OPT_ST7_VARIANT:
            if (value != 0 && !lookup7(p->dtype, p->exact, 1, value / 1000 % 10, value % 1000,
                                       std::max(1, value / 10000 % 10), value / 100000))
                return fail(ST_EINVAL, "ST_OPT_ST7_VARIANT %d is not compiled", value);
            p->opt_st7_variant = value;
            p->geo7.clear();
            return ST_OK;
        default: return fail(ST_EINVAL, "unknown option %d", option);
    }
}

extern "C" int st_plan_set_bitexact(st_plan* p, int on) {
    if (!p) return fail(ST_EINVAL, "NULL plan");
    p->exact = on != 0;
    return ST_OK;
}

static int poll_nccl(st_plan* p);

extern "C" int st_plan_sync(st_plan* p) {
    if (!p) return fail(ST_EINVAL, "NULL plan");
    CUDA_TRY(cudaStreamSynchronize(p->stream));
    CUDA_TRY(cudaGetLastError());
    return poll_nccl(p);
}

extern "C" int st_plan_ghost_planes(const st_plan* p) { return p ? p->dimT : ST_EINVAL; }

extern "C" int st_plan_local_slab(const st_plan* p, int* z0, int* nzl) {
    if (!p) return fail(ST_EINVAL, "NULL plan");
    if (z0) *z0 = p->dist.z0;
    if (nzl) *nzl = p->dist.nzl;
    return ST_OK;
}

extern "C" int st_plan_last_launches(const st_plan* p) { return p ? p->launches : ST_EINVAL; }

extern "C" int st_plan_get_info(const st_plan* p, int lbm, st_plan_info* info) {
    if (!p || !info) return fail(ST_EINVAL, "NULL argument");
    memset(info, 0, sizeof *info);
    if (lbm) {
        const int d = max_lbm_depth(p);
        GeoL g;
        if (planL(p, d, g)) return ST_EUNSUPPORTED;
        info->tile_x = 32; info->tile_y = g.TY; info->out_x = g.wx; info->out_y = g.wy;
        info->tiles_x = g.tiles_x; info->tiles_y = g.tiles_y; info->ctas = p->sms; info->threads = 32 * g.TY;
        info->smem_bytes = (int)g.smem;
        info->kappa = (double)g.tiles_x * 32 * g.tiles_y * g.TY / ((double)p->nx * p->ny);
        info->kernel = p->last_lbm_kernel ? p->last_lbm_kernel : (lbm_use_push(p) ? 100 : 200 + d);
        info->dim_t_sweep = d;
        return ST_OK;
    }
    Geo7* gp = nullptr;   // geometry of the plan's sweep depth (built on demand)
    int rc = get_geo7(const_cast<st_plan*>(p), p->dimK, p->dist.nzl, gp);
    if (rc) return rc;
    const Geo7& g = *gp;
    info->tile_x = g.TX; info->tile_y = g.TY; info->out_x = g.wx; info->out_y = g.wy;
    info->tiles_x = g.tiles_x; info->tiles_y = g.tiles_y; info->ctas = g.grid; info->threads = g.threads;
    info->smem_bytes = (int)g.smem; info->kappa = g.kappa;
    info->kernel = g.vxk * 100000 + g.minb * 10000 + g.VY * 1000 + g.maxt;
    info->dim_t_sweep = p->dimK;
    info->ring = g.ring;
    return ST_OK;
}

// ----------------------------------------------------------------------------
// helpers
// ----------------------------------------------------------------------------
static int ptr_kind(const void* ptr) {  // 1 device, 0 host, -1 error
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, ptr) != cudaSuccess) { cudaGetLastError(); return 0; }
    return (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) ? 1 : 0;
}

static int ensure_hbuf(st_plan* p, size_t bytes) {
    if (p->hbuf_bytes >= bytes) return ST_OK;
    for (void*& b : p->hbuf) { if (b) cudaFree(b); b = nullptr; }
    p->hbuf_bytes = 0;
    for (void*& b : p->hbuf)
        if (cudaMalloc(&b, bytes) != cudaSuccess) { cudaGetLastError(); return fail(ST_ENOMEM, "device staging %zu B", bytes); }
    p->hbuf_bytes = bytes;
    return ST_OK;
}

// depths of the sweeps: S = ceil(T/dim_T) sweeps, made odd so the result
// lands in `out` (ping-pong); depths as equal as possible, each <= dim_T
static std::vector<int> sweep_depths(int T, int D) {
    std::vector<int> v;
    if (T <= 0) return v;
    int S = (T + D - 1) / D;
    if (S % 2 == 0 && S < T) ++S;
    const int q = T / S, rem = T % S;
    for (int s = 0; s < S; ++s) v.push_back(q + (s < rem ? 1 : 0));
    return v;
}

static bool overlap(const void* a, const void* b, size_t n) {
    auto x = reinterpret_cast<uintptr_t>(a), y = reinterpret_cast<uintptr_t>(b);
    return x < y + n && y < x + n;
}

// ----------------------------------------------------------------------------
// 7-point
// ----------------------------------------------------------------------------
// Flexible load balance over persistent CTAs: the (tile, plane)
// work items, in tile-major order, are cut into G contiguous ranges of equal
// COST, where a range pays its planes plus a fixed overhead per tile segment it
// touches (the 2*dim_T prolog/epilog rounds that fill and drain the on-chip
// levels, which run only some levels, plus the first plane's load latency;
// calibrated by measurement below).  Minimises the largest cost by bisection
// over a greedy cut.
static void split_work(int ntiles, int nzo, int d, int G, int* split, int zchunk = 0) {
    const long long work = (long long)ntiles * nzo;
    // per-segment restart cost in plane-equivalents: the 2d prolog rounds of a
    // segment (levels start one after another, no output) plus segment set-up
    // and first-load latency.  Measured on B200: per-CTA globaltimer trace
    // (tools/trace7.py, 256^3 FP32 d = 4): prolog 5.9 us (compile-time prolog
    // rounds; 9.8 us with checked rounds) vs 0.93 us per steady plane; A/B of
    // the constant (256^3 FP32, Gupd/s): d = 4: 4 -> 1275, 7 -> 1319,
    // 8 -> 1368, 9 -> 1405, 10 -> 1326; d = 3: 4 -> 1231, 7 -> 1256,
    // 8 -> 1308, 9 -> 1295; d = 2: 4 -> 1062, 6 -> 1151.  The spread beyond
    // the model comes from which CTAs get a second segment.
#ifdef ST_SPLIT_OVH_AB
    const long long ovh = ST_SPLIT_OVH_AB;   // A/B tuning builds only
#else
    const long long ovh = std::min(2LL * d + 2, 9LL);
#endif
    auto cuts = [&](long long C, int* out) {   // CTAs needed with per-CTA cost cap C
        if (C <= ovh) return G + 1;             // no CTA could take a plane
        long long it = 0;
        int b = 0;
        while (it < work) {
            if (out) out[b] = (int)it;
            ++b;
            long long budget = C;
            while (it < work) {
                long long in_tile = (it / nzo + 1) * nzo - it;
                if (zchunk > 0) in_tile = std::min(in_tile, zchunk - (it % nzo) % zchunk);   // a 3D block
                if (budget <= ovh) break;
                const long long take = std::min(in_tile, budget - ovh);
                it += take;
                budget -= take + ovh;
                if (take < in_tile) break;
            }
        }
        return b;
    };
    long long lo = 1, hi = work + ovh * (ntiles + 1);
    while (lo < hi) {
        const long long mid = (lo + hi) / 2;
        if (cuts(mid, nullptr) <= G) hi = mid; else lo = mid + 1;
    }
    const int used = cuts(lo, split);
    for (int b = used; b <= G; ++b) split[b] = (int)work;   // idle CTAs (tiny grids) get empty ranges
}

static int launch7(st_plan* p, const void* src, void* dst, int d, double alpha, double beta, const SlabView& sv) {
    NvtxRange nvtx_("st7 sweep");
    Geo7* g = nullptr;
    int rc = get_geo7(p, d, sv.zb - sv.za, g);
    if (rc) return rc;
    CUtensorMap map;
    rc = encode_3d(&map, src, p->dtype, p->nx, p->ny, sv.nzb, g->TX, g->TY);
    if (rc) return rc;
    St7Params prm{};
    prm.out = dst;
    prm.nx = p->nx; prm.ny = p->ny; prm.nzb = sv.nzb; prm.zbase = sv.zbase; prm.nzg = p->nz;
    prm.za = sv.za; prm.zb = sv.zb;
    prm.tiles_x = g->tiles_x; prm.ntiles = g->tiles_x * g->tiles_y;
    prm.wx = g->wx; prm.wy = g->wy; prm.hx = g->hx;
    prm.tiles_y = g->tiles_y; prm.ey = g->ey; prm.ly_last = g->ly_last; prm.oy0_last = g->oy0_last;
    prm.ring = g->ring;
    prm.pdl = p->opt_pdl;
    prm.zchunk = p->opt_zchunk;
    prm.alpha = alpha; prm.beta = beta;
    if ((long long)prm.ntiles * (sv.zb - sv.za) <= 0) return ST_OK;
    if ((long long)prm.ntiles * (sv.zb - sv.za) >= (1LL << 31)) return fail(ST_EUNSUPPORTED, "grid too large");
    const int grid = std::min(sv.grid_cap > 0 ? std::min(g->grid, sv.grid_cap) : g->grid, ST7_MAX_GRID);
    split_work(prm.ntiles, sv.zb - sv.za, d, grid, prm.split, p->opt_zchunk);
    cudaError_t e = g->fn(&map, prm, grid, g->threads, g->smem, sv.stream ? sv.stream : p->stream);
    if (e != cudaSuccess) return fail(ST_ECUDA, "st7 launch (d=%d): %s", d, cudaGetErrorString(e));
    ++p->launches;
    return ST_OK;
}

// ----------------------------------------------------------------------------
// multi-sweep driver over the plan's Z decomposition (dist.h)
// ----------------------------------------------------------------------------
// ncomp: SoA components of a cell (1 for the 7-point grid, 19 for D3Q19); each
// component of a slab buffer is nzb consecutive planes.
// asynchronous NCCL errors (a peer died, a network error) surface as ST_ENCCL
// at the end of every distributed run and at st_plan_sync
static int poll_nccl(st_plan* p) {
#if ST_HAVE_NCCL
    if (p->dist.mode != Dist::NCCL || !p->dist.nccl_comm || !nccl().commGetAsyncError) return ST_OK;
    ncclResult_t ae = ncclSuccess;
    ncclResult_t r = nccl().commGetAsyncError(p->dist.nccl_comm, &ae);
    if (r != ncclSuccess) return fail(ST_ENCCL, "ncclCommGetAsyncError: %s", nccl().errorString(r));
    if (ae != ncclSuccess && ae != ncclInProgress) return fail(ST_ENCCL, "NCCL async error: %s", nccl().errorString(ae));
#else
    (void)p;
#endif
    return ST_OK;
}

static int exchange_nccl(st_plan* p, void* buf, int d, int ncomp, cudaStream_t st) {
    NvtxRange nvtx_("ghost exchange");
#if ST_HAVE_NCCL
    Dist& D = p->dist;
    const size_t pb = (size_t)p->nx * p->ny * esize(p->dtype);
    const size_t cs = (size_t)D.nzb * pb;
    char* b = static_cast<char*>(buf);
    const size_t bytes = (size_t)d * pb;
    auto& N = nccl();
    ncclResult_t r = N.groupStart();
    for (int c = 0; c < ncomp && r == ncclSuccess; ++c) {
        char* base = b + c * cs;
        if (D.rank > 0) {
            if (r == ncclSuccess) r = N.send(base + (size_t)D.g * pb, bytes, ncclUint8, D.rank - 1, D.nccl_comm, st);
            if (r == ncclSuccess) r = N.recv(base + (size_t)(D.g - d) * pb, bytes, ncclUint8, D.rank - 1, D.nccl_comm, st);
        }
        if (D.rank < D.P - 1) {
            if (r == ncclSuccess) r = N.send(base + (size_t)(D.g + D.nzl - d) * pb, bytes, ncclUint8, D.rank + 1, D.nccl_comm, st);
            if (r == ncclSuccess) r = N.recv(base + (size_t)(D.g + D.nzl) * pb, bytes, ncclUint8, D.rank + 1, D.nccl_comm, st);
        }
    }
    ncclResult_t r2 = N.groupEnd();
    if (r != ncclSuccess || r2 != ncclSuccess)
        return fail(ST_ENCCL, "ghost exchange: %s", N.errorString(r != ncclSuccess ? r : r2));
    return ST_OK;
#else
    (void)p; (void)buf; (void)d; (void)ncomp; (void)st;
    return fail(ST_EUNSUPPORTED, "built without NCCL");
#endif
}

static int exchange_loop(st_plan* p, int cur, int d, int ncomp, cudaStream_t st) {
    Dist& D = p->dist;
    const size_t pb = (size_t)p->nx * p->ny * esize(p->dtype);
    const size_t bytes = (size_t)d * pb;
    for (int k = 0; k < D.P; ++k) {
        Dist::Slab& s = D.slabs[k];
        char* me = static_cast<char*>(s.buf[cur]);
        const size_t cs = (size_t)s.nzb * pb;
        if (k > 0) {
            Dist::Slab& o = D.slabs[k - 1];
            const char* src = static_cast<const char*>(o.buf[cur]);
            const size_t ocs = (size_t)o.nzb * pb;
            for (int c = 0; c < ncomp; ++c)
                CUDA_TRY(cudaMemcpyAsync(me + c * cs + (size_t)(D.g - d) * pb,
                                         src + c * ocs + (size_t)(D.g + o.nzl - d) * pb, bytes,
                                         cudaMemcpyDeviceToDevice, st));
        }
        if (k < D.P - 1) {
            Dist::Slab& o = D.slabs[k + 1];
            const char* src = static_cast<const char*>(o.buf[cur]);
            const size_t ocs = (size_t)o.nzb * pb;
            for (int c = 0; c < ncomp; ++c)
                CUDA_TRY(cudaMemcpyAsync(me + c * cs + (size_t)(D.g + s.nzl) * pb, src + c * ocs + (size_t)D.g * pb,
                                         bytes, cudaMemcpyDeviceToDevice, st));
        }
    }
    return ST_OK;
}

// copy global planes [z, z+n) of every component between a full grid (nz planes)
// and a slab buffer (nzb planes, buffer plane = z - zbase)
static int slab_copy(st_plan* p, void* full, void* slab, int zbase, int nzb, int z, int n, int ncomp, bool to_slab) {
    if (n <= 0) return ST_OK;
    const size_t pb = (size_t)p->nx * p->ny * esize(p->dtype);
    for (int c = 0; c < ncomp; ++c) {
        char* f = static_cast<char*>(full) + (size_t)c * p->nz * pb + (size_t)z * pb;
        char* s = static_cast<char*>(slab) + (size_t)c * nzb * pb + (size_t)(z - zbase) * pb;
        CUDA_TRY(cudaMemcpyAsync(to_slab ? s : f, to_slab ? f : s, (size_t)n * pb, cudaMemcpyDeviceToDevice,
                                 p->stream));
    }
    return ST_OK;
}

static int ensure_loop_slabs(st_plan* p, int ncomp, const uint8_t* flags) {
    Dist& D = p->dist;
    const size_t pbe = (size_t)p->nx * p->ny * esize(p->dtype);
    const size_t plane = (size_t)p->nx * p->ny;
    for (auto& s : D.slabs) {
        const size_t need = (size_t)ncomp * s.nzb * pbe;
        if (D.slab_cell_bytes < need / s.nzb / plane * 1 || D.slab_ncomp != ncomp || !s.buf[0]) {
            for (void*& b : s.buf) { if (b) cudaFree(b); b = nullptr; }
            for (void*& b : s.buf)
                if (cudaMalloc(&b, need) != cudaSuccess) { cudaGetLastError(); return fail(ST_ENOMEM, "loopback slab"); }
        }
        if (flags) {
            if (!s.flags && cudaMalloc(&s.flags, (size_t)s.nzb * plane) != cudaSuccess) return fail(ST_ENOMEM, "slab flags");
            if (!s.fl2 && cudaMalloc(&s.fl2, (size_t)s.nzb * plane) != cudaSuccess) return fail(ST_ENOMEM, "slab fl2");
            // planes outside the lattice are WALL; the rest copied from the global flags
            CUDA_TRY(cudaMemsetAsync(s.flags, ST_WALL, (size_t)s.nzb * plane, p->stream));
            const int zlo = std::max(0, s.z0 - D.g), zhi = std::min(p->nz, s.z0 + s.nzl + D.g);
            CUDA_TRY(cudaMemcpyAsync(s.flags + (size_t)(zlo - (s.z0 - D.g)) * plane, flags + (size_t)zlo * plane,
                                     (size_t)(zhi - zlo) * plane, cudaMemcpyDeviceToDevice, p->stream));
            cudaError_t e = lbm_fl2(s.flags, s.fl2, p->nx, p->ny, s.nzb, p->stream);
            if (e != cudaSuccess) return fail(ST_ECUDA, "slab fl2: %s", cudaGetErrorString(e));
        }
    }
    D.slab_ncomp = ncomp;
    D.slab_cell_bytes = (size_t)ncomp * esize(p->dtype);
    return ST_OK;
}

static int ensure_comm(st_plan* p) {
    Dist& D = p->dist;
    if (!D.comm) CUDA_TRY(cudaStreamCreateWithFlags(&D.comm, cudaStreamNonBlocking));
    if (!D.ev_b) CUDA_TRY(cudaEventCreateWithFlags(&D.ev_b, cudaEventDisableTiming));
    if (!D.ev_x) CUDA_TRY(cudaEventCreateWithFlags(&D.ev_x, cudaEventDisableTiming));
    return ST_OK;
}

// Sweeps over Z slabs with the ghost exchange for sweep k+1 overlapped with
// the interior of sweep k: the d' output planes next to each
// slab face are computed first, an event hands them to the exchange stream,
// the interior planes are computed meanwhile, and sweep k+1 waits for the
// exchange.  ST_OPT_OVERLAP = 0 serialises exchange and sweep (A/B).
template <typename L>
static int run_sweeps(st_plan* p, const std::vector<int>& ds, const void* in, void* out, int ncomp,
                      const uint8_t* flags, L&& launch) {
    Dist& D = p->dist;
    const size_t pb = (size_t)p->nx * p->ny * esize(p->dtype);
    const bool overlap_ok = p->opt_overlap != 0;
    if (D.mode == Dist::SINGLE) {
        const void* src = in;
        void* dst = out;
        void* bufs[2] = {const_cast<void*>(in), out};
        for (size_t k = 0; k < ds.size(); ++k) {
            SlabView sv;
            sv.stream = p->stream; sv.flags = flags; sv.fl2 = p->fl2;
            sv.nzb = p->nz; sv.zbase = 0; sv.za = 0; sv.zb = p->nz; sv.single = true; sv.sweep = (int)k;
            int rc = launch(src, dst, ds[k], sv);
            if (rc) return rc;
            src = bufs[(k + 1) % 2];
            dst = bufs[k % 2];
        }
        if (ds.size() % 2 == 0)  // only when every sweep has depth 1 and T is even: result in `in`
            CUDA_TRY(cudaMemcpyAsync(out, in, (size_t)ncomp * D.nzb * pb, cudaMemcpyDeviceToDevice, p->stream));
        return ST_OK;
    }
    int rc = ensure_comm(p);
    if (rc) return rc;
    const bool loop = D.mode == Dist::LOOPBACK;
    // slab list: loopback = every virtual slab; NCCL = this rank's slab in the caller's buffers
    struct S { void* buf[2]; int z0, nzl, nzb; const uint8_t* flags; uint8_t* fl2; };
    std::vector<S> sl;
    if (loop) {
        rc = ensure_loop_slabs(p, ncomp, flags);
        if (rc) return rc;
        for (auto& s : D.slabs) {   // scatter owned planes + available ghosts
            const int zlo = std::max(0, s.z0 - D.g), zhi = std::min(p->nz, s.z0 + s.nzl + D.g);
            rc = slab_copy(p, const_cast<void*>(in), s.buf[0], s.z0 - D.g, s.nzb, zlo, zhi - zlo, ncomp, true);
            if (rc) return rc;
            sl.push_back({{s.buf[0], s.buf[1]}, s.z0, s.nzl, s.nzb, s.flags, s.fl2});
        }
    } else {
        sl.push_back({{const_cast<void*>(in), out}, D.z0, D.nzl, D.nzb, flags, p->fl2});
    }
    auto exchange = [&](int which, int d, cudaStream_t st) -> int {
        if (loop) return exchange_loop(p, which, d, ncomp, st);
        return exchange_nccl(p, sl[0].buf[which], d, ncomp, st);
    };
    auto view = [&](const S& s, int za, int zb, int cap, int sweep) {
        SlabView sv;
        sv.sweep = sweep;
        sv.nzb = s.nzb; sv.zbase = s.z0 - D.g; sv.za = za; sv.zb = zb;
        sv.flags = s.flags; sv.fl2 = s.fl2; sv.single = false; sv.stream = p->stream; sv.grid_cap = cap;
        return sv;
    };
    // the schedule (dist.h slab_schedule, also exported as st_slab_schedule) is
    // identical for every slab up to its plane count; run step by step over all slabs
    int nzl_min = sl[0].nzl;
    for (auto& s : sl) nzl_min = std::min(nzl_min, s.nzl);
    std::vector<std::vector<SlabStep>> sched;
    for (auto& s : sl) sched.push_back(slab_schedule(ds, D.g, s.nzl, nzl_min, overlap_ok));
    const int cap = loop ? 0 : std::max(1, p->sms - 8);   // leave SMs to the NCCL kernels
    int cur = 0;
    for (size_t i = 0; i < sched[0].size(); ++i) {
        const SlabStep& st0 = sched[0][i];
        switch (st0.kind) {
            case SlabStep::EXCHANGE:
                if (st0.async) {
                    CUDA_TRY(cudaEventRecord(D.ev_b, p->stream));
                    CUDA_TRY(cudaStreamWaitEvent(D.comm, D.ev_b, 0));
                    rc = exchange(st0.src, st0.depth, D.comm);
                    if (rc) return rc;
                    CUDA_TRY(cudaEventRecord(D.ev_x, D.comm));
                } else {
                    rc = exchange(st0.src, st0.depth, p->stream);
                    if (rc) return rc;
                }
                break;
            case SlabStep::SWEEP:
                for (size_t k = 0; k < sl.size(); ++k) {
                    const SlabStep& stp = sched[k][i];
                    rc = launch(sl[k].buf[stp.src], sl[k].buf[1 - stp.src], stp.depth,
                                view(sl[k], stp.z_begin, stp.z_end, stp.grid_cap ? cap : 0, stp.sweep));
                    if (rc) return rc;
                }
                cur = 1 - st0.src;
                break;
            case SlabStep::WAIT:
                CUDA_TRY(cudaStreamWaitEvent(p->stream, D.ev_x, 0));
                break;
            case SlabStep::COPY:
                cur = 0;
                break;
        }
    }
    rc = poll_nccl(p);
    if (rc) return rc;
    if (loop) {
        for (auto& s : D.slabs) {   // gather owned planes
            rc = slab_copy(p, out, cur == 0 ? s.buf[0] : s.buf[1], s.z0 - D.g, s.nzb, s.z0, s.nzl, ncomp, false);
            if (rc) return rc;
        }
    } else if (cur == 0) {   // even number of sweeps (the schedule's COPY): the result is in `in`
        CUDA_TRY(cudaMemcpyAsync(out, in, (size_t)ncomp * D.nzb * pb, cudaMemcpyDeviceToDevice, p->stream));
    }
    return ST_OK;
}

static int run7_device(st_plan* p, const void* in, void* out, double alpha, double beta, int T) {
    const size_t n = (size_t)p->nx * p->ny * p->dist.nzb * esize(p->dtype);
    p->launches = 0;
    if (T == 0) {
        CUDA_TRY(cudaMemcpyAsync(out, in, n, cudaMemcpyDeviceToDevice, p->stream));
        return ST_OK;
    }
    if (p->variant == ST_VARIANT_NAIVE) {   // ablation baseline: T single-step launches, ping-pong
        if (p->dist.mode != Dist::SINGLE) return fail(ST_EUNSUPPORTED, "the naive variant is single-process only");
        const void* src = in;
        void* bufs[2] = {const_cast<void*>(in), out};
        for (int k = 0; k < T; ++k) {
            void* dst = bufs[(k + 1) % 2];
            cudaError_t e = st7_naive_launch(p->dtype == ST_F32 ? 0 : 1, src, dst, p->nx, p->ny, p->nz, alpha, beta,
                                             p->stream);
            if (e != cudaSuccess) return fail(ST_ECUDA, "naive launch: %s", cudaGetErrorString(e));
            ++p->launches;
            src = dst;
        }
        if (T % 2 == 0) CUDA_TRY(cudaMemcpyAsync(out, in, n, cudaMemcpyDeviceToDevice, p->stream));
        return ST_OK;
    }
    std::vector<int> ds = sweep_depths(T, p->dimK);
    int rc = run_sweeps(p, ds, in, out, 1, nullptr, [&](const void* a, void* b, int d, const SlabView& sv) {
        return launch7(p, a, b, d, alpha, beta, sv);
    });
    if (rc) return rc;
    CUDA_TRY(cudaGetLastError());
    return ST_OK;
}

extern "C" int st7_run(st_plan* p, const void* in, void* out, double alpha, double beta, int T) {
    NvtxRange nvtx_("st7_run");
    if (!p) return fail(ST_EINVAL, "NULL plan");
    if (!in || !out) return fail(ST_EINVAL, "NULL grid pointer");
    if (T < 0) return fail(ST_EINVAL, "T = %d < 0", T);
    const size_t n = (size_t)p->nx * p->ny * p->dist.nzb * esize(p->dtype);
    if (overlap(in, out, n)) return fail(ST_EINVAL, "in and out overlap");
    const int kin = ptr_kind(in), kout = ptr_kind(out);
    if (kin != kout) return fail(ST_EINVAL, "in and out must both be host or both be device pointers");
    if (kin == 1) {
        if ((reinterpret_cast<uintptr_t>(in) | reinterpret_cast<uintptr_t>(out)) & 15)
            return fail(ST_EINVAL, "device grids must be 16-byte aligned");
        return run7_device(p, in, out, alpha, beta, T);
    }
    // host pointers: stage through plan-owned device buffers, synchronous
    int rc = ensure_hbuf(p, n);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(p->hbuf[0], in, n, cudaMemcpyHostToDevice, p->stream));
    rc = run7_device(p, p->hbuf[0], p->hbuf[1], alpha, beta, T);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(out, p->hbuf[1], n, cudaMemcpyDeviceToHost, p->stream));
    CUDA_TRY(cudaStreamSynchronize(p->stream));
    return ST_OK;
}

// ----------------------------------------------------------------------------
// 27-point stencil: ceil(T/D) ping-pong sweeps of the
// st27.cu kernel, D = min(dim_T, st27_depth_max()); single process only.
// ----------------------------------------------------------------------------
static int launch27t(st_plan* p, const void* src, void* dst, int d, const double w[4]) {
    NvtxRange nvtx_("st27 sweep");
    Geo7 g;
    int rc = plan27t(p, d, p->nz, g);
    if (rc) return rc;
    CUtensorMap map;
    rc = encode_3d(&map, src, p->dtype, p->nx, p->ny, p->nz, g.TX, g.TY);
    if (rc) return rc;
    St27tParams prm{};
    St7Params& q = prm.g;
    q.out = dst;
    q.nx = p->nx; q.ny = p->ny; q.nzb = p->nz; q.zbase = 0; q.nzg = p->nz;
    q.za = 0; q.zb = p->nz;
    q.tiles_x = g.tiles_x; q.ntiles = g.tiles_x * g.tiles_y;
    q.wx = g.wx; q.wy = g.wy; q.hx = g.hx;
    q.tiles_y = g.tiles_y; q.ey = g.ey; q.ly_last = g.ly_last; q.oy0_last = g.oy0_last;
    q.ring = g.ring;
    q.pdl = p->opt_pdl;
    q.alpha = w[0]; q.beta = w[1]; prm.gamma = w[2]; prm.delta = w[3];
    if ((long long)q.ntiles * p->nz >= (1LL << 31)) return fail(ST_EUNSUPPORTED, "grid too large");
    const int grid = std::min(g.grid, ST7_MAX_GRID);
    split_work(q.ntiles, p->nz, d, grid, q.split);   // restart: 2d-1 prolog rounds
    cudaError_t e = g.fn27t(&map, prm, grid, g.threads, g.smem, p->stream);
    if (e != cudaSuccess) return fail(ST_ECUDA, "st27t launch (d=%d): %s", d, cudaGetErrorString(e));
    ++p->launches;
    return ST_OK;
}

static int run27_device(st_plan* p, const void* in, void* out, const double w[4], int T) {
    const size_t n = (size_t)p->nx * p->ny * p->nz * esize(p->dtype);
    p->launches = 0;
    if (T == 0) {
        CUDA_TRY(cudaMemcpyAsync(out, in, n, cudaMemcpyDeviceToDevice, p->stream));
        return ST_OK;
    }
    // tolerance build: the 7-point machinery (st27t); bit-exact build: the oracle-order kernel (st27.cu)
    const bool tk = !p->exact;
    const int D = std::min(p->dimT, tk ? ST27T_MAX_DIM_T : st27_depth_max(p->dtype == ST_F32 ? 0 : 1));
    const std::vector<int> ds = sweep_depths(T, D);
    void* bufs[2] = {const_cast<void*>(in), out};
    for (size_t k = 0; k < ds.size(); ++k) {
        if (tk) {
            int rc = launch27t(p, bufs[k % 2], bufs[(k + 1) % 2], ds[k], w);
            if (rc) return rc;
            continue;
        }
        cudaError_t e = st27_launch(p->dtype == ST_F32 ? 0 : 1, p->exact, ds[k], bufs[k % 2], bufs[(k + 1) % 2], p->nx,
                                    p->ny, p->nz, w[0], w[1], w[2], w[3], p->sms, p->stream, nullptr);
        if (e != cudaSuccess) return fail(ST_ECUDA, "st27 launch: %s", cudaGetErrorString(e));
        ++p->launches;
    }
    if (ds.size() % 2 == 0) CUDA_TRY(cudaMemcpyAsync(out, in, n, cudaMemcpyDeviceToDevice, p->stream));
    return ST_OK;
}

extern "C" int st27_run(st_plan* p, const void* in, void* out, double alpha, double beta, double gamma, double delta,
                        int T) {
    NvtxRange nvtx_("st27_run");
    if (!p) return fail(ST_EINVAL, "NULL plan");
    if (!in || !out) return fail(ST_EINVAL, "NULL grid pointer");
    if (T < 0) return fail(ST_EINVAL, "T = %d < 0", T);
    if (p->dist.mode != Dist::SINGLE) return fail(ST_EUNSUPPORTED, "st27_run is single-process only");
    const size_t n = (size_t)p->nx * p->ny * p->nz * esize(p->dtype);
    if (overlap(in, out, n)) return fail(ST_EINVAL, "in and out overlap");
    const int kin = ptr_kind(in), kout = ptr_kind(out);
    if (kin != kout) return fail(ST_EINVAL, "in and out must both be host or both be device pointers");
    const double w[4] = {alpha, beta, gamma, delta};
    if (kin == 1) {
        if ((reinterpret_cast<uintptr_t>(in) | reinterpret_cast<uintptr_t>(out)) & 15)
            return fail(ST_EINVAL, "device grids must be 16-byte aligned");
        return run27_device(p, in, out, w, T);
    }
    int rc = ensure_hbuf(p, n);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(p->hbuf[0], in, n, cudaMemcpyHostToDevice, p->stream));
    rc = run27_device(p, p->hbuf[0], p->hbuf[1], w, T);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(out, p->hbuf[1], n, cudaMemcpyDeviceToHost, p->stream));
    CUDA_TRY(cudaStreamSynchronize(p->stream));
    return ST_OK;
}

// ----------------------------------------------------------------------------
// Radius-2 13-point star (general R of §V; X25/X26):
// ceil(T/D) ping-pong sweeps of st13_kernel.cuh, D = min(dim_T, 4 FP32 / 3 FP64); single
// process only.
// ----------------------------------------------------------------------------
static int launch13(st_plan* p, const void* src, void* dst, int d, const double w[3]) {
    NvtxRange nvtx_("st13 sweep");
    Geo7 g;
    int rc = plan13(p, d, p->nz, g);
    if (rc) return rc;
    CUtensorMap map;
    rc = encode_3d(&map, src, p->dtype, p->nx, p->ny, p->nz, g.TX, g.TY);
    if (rc) return rc;
    St13Params prm{};
    St7Params& q = prm.g;
    q.out = dst;
    q.nx = p->nx; q.ny = p->ny; q.nzb = p->nz; q.zbase = 0; q.nzg = p->nz;
    q.za = 0; q.zb = p->nz;
    q.tiles_x = g.tiles_x; q.ntiles = g.tiles_x * g.tiles_y;
    q.wx = g.wx; q.wy = g.wy; q.hx = g.hx;
    q.tiles_y = g.tiles_y; q.ey = g.ey; q.ly_last = g.ly_last; q.oy0_last = g.oy0_last;
    q.ring = g.ring;
    q.pdl = p->opt_pdl;
    q.alpha = w[0]; q.beta = w[1]; prm.gamma = w[2];
    if ((long long)q.ntiles * p->nz >= (1LL << 31)) return fail(ST_EUNSUPPORTED, "grid too large");
    const int grid = std::min(g.grid, ST7_MAX_GRID);
    split_work(q.ntiles, p->nz, 2 * d, grid, q.split);
    cudaError_t e = g.fn13(&map, prm, grid, g.threads, g.smem, p->stream);
    if (e != cudaSuccess) return fail(ST_ECUDA, "st13 launch (d=%d): %s", d, cudaGetErrorString(e));
    ++p->launches;
    return ST_OK;
}

static int run13_device(st_plan* p, const void* in, void* out, const double w[3], int T) {
    const size_t n = (size_t)p->nx * p->ny * p->nz * esize(p->dtype);
    p->launches = 0;
    if (T == 0) {
        CUDA_TRY(cudaMemcpyAsync(out, in, n, cudaMemcpyDeviceToDevice, p->stream));
        return ST_OK;
    }
    // FP64 at depth 4 needs 16 halo rows per side: no 256-thread tile fits
    const std::vector<int> ds = sweep_depths(T, std::min(p->dimT, p->dtype == ST_F32 ? ST13_MAX_DIM_T : 3));
    void* bufs[2] = {const_cast<void*>(in), out};
    for (size_t k = 0; k < ds.size(); ++k) {
        int rc = launch13(p, bufs[k % 2], bufs[(k + 1) % 2], ds[k], w);
        if (rc) return rc;
    }
    if (ds.size() % 2 == 0) CUDA_TRY(cudaMemcpyAsync(out, in, n, cudaMemcpyDeviceToDevice, p->stream));
    CUDA_TRY(cudaGetLastError());
    return ST_OK;
}

extern "C" int st13_run(st_plan* p, const void* in, void* out, double alpha, double beta, double gamma, int T) {
    NvtxRange nvtx_("st13_run");
    if (!p) return fail(ST_EINVAL, "NULL plan");
    if (!in || !out) return fail(ST_EINVAL, "NULL grid pointer");
    if (T < 0) return fail(ST_EINVAL, "T = %d < 0", T);
    if (p->dist.mode != Dist::SINGLE) return fail(ST_EUNSUPPORTED, "st13_run is single-process only");
    if (p->nx < 5 || p->ny < 5 || p->nz < 5) return fail(ST_EINVAL, "radius 2 needs every extent >= 5");
    const size_t n = (size_t)p->nx * p->ny * p->nz * esize(p->dtype);
    if (overlap(in, out, n)) return fail(ST_EINVAL, "in and out overlap");
    const int kin = ptr_kind(in), kout = ptr_kind(out);
    if (kin != kout) return fail(ST_EINVAL, "in and out must both be host or both be device pointers");
    const double w[3] = {alpha, beta, gamma};
    if (kin == 1) {
        if ((reinterpret_cast<uintptr_t>(in) | reinterpret_cast<uintptr_t>(out)) & 15)
            return fail(ST_EINVAL, "device grids must be 16-byte aligned");
        return run13_device(p, in, out, w, T);
    }
    int rc = ensure_hbuf(p, n);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(p->hbuf[0], in, n, cudaMemcpyHostToDevice, p->stream));
    rc = run13_device(p, p->hbuf[0], p->hbuf[1], w, T);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(out, p->hbuf[1], n, cudaMemcpyDeviceToHost, p->stream));
    CUDA_TRY(cudaStreamSynchronize(p->stream));
    return ST_OK;
}

// ----------------------------------------------------------------------------
// Blocking-parameter selection ("a framework that determines the
// various blocking parameters"; eqs. (1)-(4)): the eq. (3) bound
// eta, the smallest depth with dim_T / kappa > gamma / Gamma (eq. (3)
// with the overestimation kappa of the planner's tiling, eq. (2)), evaluated
// with a Gamma MEASURED on this device and kernel -- the bytes/s of a depth-1
// sweep (the bandwidth the kernel gets) over the FP lane-ops/s of the
// deepest sweep (the rate its issue-limited compute reaches, ghost points
// included) -- seeds the search; depths eta-1..eta+1 are timed and the
// search walks on while a neighbour is faster, so the nominal-peak eta (6-7
// on B200, where the kernel is not FP-pipe bound) never costs 8 timings.
// ----------------------------------------------------------------------------
static int time_depth(st_plan* p, void* a, void* b, int d, int T_probe, cudaEvent_t e0, cudaEvent_t e1, float& ms) {
    p->dimK = d;
    int rc = run7_device(p, a, b, 0.4, 0.1, std::min(T_probe, 2 * d));   // warm-up (geometry, first launch)
    if (rc) return rc;
    cudaEventRecord(e0, p->stream);
    rc = run7_device(p, a, b, 0.4, 0.1, T_probe);
    if (rc) return rc;
    cudaEventRecord(e1, p->stream);
    if (cudaEventSynchronize(e1) != cudaSuccess) return fail(ST_ECUDA, "autotune: %s", cudaGetErrorString(cudaGetLastError()));
    cudaEventElapsedTime(&ms, e0, e1);
    return ST_OK;
}

extern "C" int st_plan_autotune_report(st_plan* p, void* a, void* b, int T_probe, st_autotune_report* rep) {
    if (!p) return fail(ST_EINVAL, "NULL plan");
    if (!a || !b) return fail(ST_EINVAL, "NULL grid pointer");
    if (T_probe < 1) return fail(ST_EINVAL, "T_probe = %d < 1", T_probe);
    if (p->dist.mode != Dist::SINGLE) return fail(ST_EUNSUPPORTED, "autotune a single-process plan and broadcast");
    const size_t n = (size_t)p->nx * p->ny * p->dist.nzb * esize(p->dtype);
    if (overlap(a, b, n)) return fail(ST_EINVAL, "a and b overlap");
    if (ptr_kind(a) != 1 || ptr_kind(b) != 1) return fail(ST_EINVAL, "autotune needs device grids");
    if ((reinterpret_cast<uintptr_t>(a) | reinterpret_cast<uintptr_t>(b)) & 15)
        return fail(ST_EINVAL, "device grids must be 16-byte aligned");
    st_autotune_report r;
    memset(&r, 0, sizeof r);
    const double E = (double)esize(p->dtype);
    r.gamma = 2.0 * E / 7.0;                         // bytes per FP lane-op of the 7-point update
    {   // nominal Gamma: device HBM bytes/s over FP lane-ops/s (FP32 128 / FP64 64 lanes per SM)
        int memclk_khz = 0, bus_bits = 0, smclk_khz = 0;
        cudaDeviceGetAttribute(&memclk_khz, cudaDevAttrMemoryClockRate, p->dev);
        cudaDeviceGetAttribute(&bus_bits, cudaDevAttrGlobalMemoryBusWidth, p->dev);
        cudaDeviceGetAttribute(&smclk_khz, cudaDevAttrClockRate, p->dev);
        const double lanes = p->dtype == ST_F32 ? 128.0 : 64.0;
        const double bw = 2.0 * memclk_khz * 1e3 * bus_bits / 8.0;
        const double ops = (double)p->sms * lanes * smclk_khz * 1e3;
        r.Gamma_nominal = (bw > 0 && ops > 0) ? bw / ops : 0;
        st_blocking m{};
        r.eta_nominal = r.Gamma_nominal > 0 && st_blocking_model(p->smem_optin, E, 1, r.gamma, r.Gamma_nominal, 0, 0, &m) == ST_OK
                            ? m.eta : 0;
    }
    cudaEvent_t e0, e1;
    CUDA_TRY(cudaEventCreate(&e0));
    CUDA_TRY(cudaEventCreate(&e1));
    const int keep = p->dimK, dmax = p->dimKmax;
    const double upd = (double)(p->nx - 2) * (p->ny - 2) * (p->nz - 2) * T_probe;
    int rc = ST_OK;
    auto probe = [&](int d) -> float {
        if (d < 1 || d > dmax) return 0.f;
        if (r.ms[d - 1] > 0) return r.ms[d - 1];
        float ms = 0.f;
        if (rc == ST_OK) rc = time_depth(p, a, b, d, T_probe, e0, e1, ms);
        if (rc == ST_OK) { r.ms[d - 1] = ms; r.tested[d - 1] = 1; }
        return rc == ST_OK ? ms : 0.f;
    };
    // measured Gamma: bytes/s at depth 1 (2E per point per sweep) over FP lane-ops/s at the deepest depth
    const float m1 = probe(1), md = probe(dmax);
    // kappa(d): loaded / useful points of the planner's tiling at depth d (eq. (2) analog)
    auto kappa_at = [&](int d) {
        Geo7* g = nullptr;
        return get_geo7(p, d, p->dist.nzl, g) == ST_OK ? g->kappa : 1.0;
    };
    if (rc == ST_OK && m1 > 0 && md > 0) {
        const double sweeps1 = (double)sweep_depths(T_probe, 1).size();
        r.bw_dim1 = 2.0 * E * (double)p->nx * p->ny * p->nz * sweeps1 / (m1 * 1e-3);
        // FP lane-ops the deepest sweep executes, redundant (ghost) points included
        r.fp_deep = 7.0 * upd * kappa_at(dmax) / (md * 1e-3);
        r.Gamma_eff = r.bw_dim1 / r.fp_deep;
        // blocking pays while dim_T / kappa > gamma / Gamma -> the smallest such depth
        r.eta = dmax;
        for (int d = 1; d <= dmax; ++d)
            if (d / kappa_at(d) >= r.gamma / r.Gamma_eff) { r.eta = d; break; }
    }
    // eq. (4) tile sides at eta for three on-chip capacities: one CTA's shared
    // memory, the SM's shared memory + register file, an 8-CTA cluster's DSMEM
    {
        int regs = 0;
        cudaDeviceGetAttribute(&regs, cudaDevAttrMaxRegistersPerMultiprocessor, p->dev);
        const double caps[3] = {(double)p->smem_optin, (double)p->smem_sm + 4.0 * regs, 8.0 * p->smem_optin};
        for (int c = 0; c < 3; ++c) {
            st_blocking m{};
            if (r.eta > 0 && st_blocking_model(caps[c], E, 1, r.gamma, r.gamma / r.eta, r.eta, 0, &m) == ST_OK) {
                r.capacity[c] = caps[c];
                r.tile_side[c] = m.dim;
                r.kappa[c] = m.kappa;
            }
        }
    }
    // seed at eta, time its neighbours, walk toward the faster side
    int best = 1;
    if (rc == ST_OK) {
        const int seed = std::max(1, std::min(r.eta > 0 ? r.eta : dmax, dmax));
        for (int d = seed - 1; d <= seed + 1; ++d) probe(d);
        auto best_tested = [&]() {
            int b = 0;
            for (int d = 1; d <= dmax; ++d)
                if (r.ms[d - 1] > 0 && (b == 0 || r.ms[d - 1] < r.ms[b - 1])) b = d;
            return b;
        };
        for (int guard = 0; guard < dmax && rc == ST_OK; ++guard) {
            best = best_tested();
            const int lo = best - 1, hi = best + 1;
            const bool more = (lo >= 1 && r.ms[lo - 1] == 0) || (hi <= dmax && r.ms[hi - 1] == 0);
            if (!more) break;
            probe(lo);
            probe(hi);
        }
        best = best_tested();
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    p->dimK = rc ? keep : best;
    r.dim_T = rc ? 0 : best;
    if (rep) *rep = r;
    return rc ? rc : best;
}

extern "C" int st_plan_autotune(st_plan* p, void* a, void* b, int T_probe, int* eta_out, float* ms_out) {
    st_autotune_report r;
    const int rc = st_plan_autotune_report(p, a, b, T_probe, &r);
    if (rc < 0) return rc;
    if (eta_out) *eta_out = r.eta;
    if (ms_out)
        for (int d = 0; d < ST_MAX_DIM_T; ++d) ms_out[d] = r.ms[d];
    return rc;
}

// ----------------------------------------------------------------------------
// LBM D3Q19
// ----------------------------------------------------------------------------
template <typename T>
static void lid_coeffs(const double lid[3], double out[19]) {
    static const int ex[19] = {0, 1, -1, 0, 0, 0, 0, 1, -1, 1, -1, 1, -1, 1, -1, 0, 0, 0, 0};
    static const int ey[19] = {0, 0, 0, 1, -1, 0, 0, 1, -1, -1, 1, 0, 0, 0, 0, 1, -1, 1, -1};
    static const int ez[19] = {0, 0, 0, 0, 0, 1, -1, 0, 0, 0, 0, 1, -1, -1, 1, 1, -1, -1, 1};
    const T u[3] = {(T)lid[0], (T)lid[1], (T)lid[2]};
    for (int i = 0; i < 19; ++i) {
        const int e[3] = {ex[i], ey[i], ez[i]};
        T eu = 0;
        bool first = true;
        for (int a = 0; a < 3; ++a) {
            if (!e[a]) continue;
            T v = e[a] > 0 ? u[a] : -u[a];
            eu = first ? v : (T)(eu + v);
            first = false;
        }
        const T w = (T)1 / (T)(i == 0 ? 3 : (i <= 6 ? 18 : 36));
        const T sixw = (T)((T)6 * w);
        out[i] = (double)(T)(sixw * eu);
    }
}

// LBM 3.5D geometry for sweep depth d: 32 x TY tiles, TY as large as the
// (d-1) three-plane assembly rings allow in shared memory (<= 16 rows)
static int planL(const st_plan* p, int d, GeoL& g) {
    const size_t E = esize(p->dtype);
    for (int ty = 16; ty >= 2; --ty) {
        const size_t smem = (size_t)(d - 1) * 3 * 19 * 34 * (ty + 2) * E;
        if (smem > p->smem_optin) continue;
        if (ty - 2 * d < 1) break;
        g.TY = ty; g.smem = smem;
        g.wx = 32 - 2 * d; g.wy = ty - 2 * d;
        g.tiles_x = (p->nx + g.wx - 1) / g.wx; g.tiles_y = (p->ny + g.wy - 1) / g.wy;
        return ST_OK;
    }
    return fail(ST_EUNSUPPORTED, "LBM dim_T %d does not fit on chip", d);
}

static int max_lbm_depth(const st_plan* p) {
    GeoL g;
    for (int d = std::min(p->dimT, LBM35_MAX_D); d >= 1; --d)
        if (planL(p, d, g) == ST_OK) return d;
    return 1;
}

static bool lbm_use_push(const st_plan* p) {
    if (p->opt_lbm_kernel == 1 || p->opt_lbm_kernel == 3) return true;
    if (p->opt_lbm_kernel == 2) return false;
    return max_lbm_depth(p) == 1;
}

static int launch_lbm35(st_plan* p, const void* src, void* dst, int d, double omega, const SlabView& sv) {
    NvtxRange nvtx_("lbm 3.5D sweep");
    GeoL g;
    int rc = planL(p, d, g);
    if (rc) return rc;
    Lbm35Params prm{};
    prm.src = src; prm.dst = dst; prm.fl2 = sv.fl2;
    prm.nx = p->nx; prm.ny = p->ny; prm.nzb = sv.nzb; prm.zbase = sv.zbase; prm.nzg = p->nz;
    prm.za = sv.za; prm.zb = sv.zb;
    prm.tiles_x = g.tiles_x; prm.wx = g.wx; prm.wy = g.wy;
    prm.work = (long long)g.tiles_x * g.tiles_y * (sv.zb - sv.za);
    prm.omega = omega;
    if (p->dtype == ST_F32) lid_coeffs<float>(p->lid, prm.lidc);
    else lid_coeffs<double>(p->lid, prm.lidc);
    if (prm.work <= 0) return ST_OK;
    int grid = (int)std::min<long long>(p->sms, prm.work);
    if (sv.grid_cap > 0) grid = std::min(grid, sv.grid_cap);
    cudaError_t e = lbm35_launch(p->dtype == ST_F32 ? 0 : 1, p->exact, d, prm, grid, 32 * g.TY, g.smem,
                                 sv.stream ? sv.stream : p->stream);
    if (e != cudaSuccess) return fail(ST_ECUDA, "lbm_35d launch (d=%d): %s", d, cudaGetErrorString(e));
    ++p->launches;
    return ST_OK;
}

static int launch_lbm(st_plan* p, const void* src, void* dst, const uint8_t* flags, double omega,
                      const SlabView& sv) {
    NvtxRange nvtx_("lbm push step");
    LbmParams prm{};
    prm.nx = p->nx; prm.ny = p->ny; prm.nzb = sv.nzb; prm.zbase = sv.zbase; prm.nzg = p->nz;
    prm.za = sv.za; prm.zb = sv.zb;
    prm.omega = omega;
    if (p->dtype == ST_F32) lid_coeffs<float>(p->lid, prm.lidc);
    else lid_coeffs<double>(p->lid, prm.lidc);
    // Z-slab views also process the ghost planes next to the output planes (push form)
    const int pa = sv.single ? sv.za : std::max(sv.za - 1, 0), pb = sv.single ? sv.zb : std::min(sv.zb + 1, sv.nzb);
    const long long cells = (long long)(pb - pa) * p->nx * p->ny;
    if (cells <= 0 || sv.zb <= sv.za) return ST_OK;
    // one wave of resident 256-thread CTAs (the kernel's launch bounds), grid-stride
    const bool batched = lbm_push_batched((int)esize(p->dtype), p->nx, p->ny, sv.nzb, p->opt_lbm_batched);
    const int bps = p->dtype == ST_F32 ? lbm_push_ctas<float>(batched) : lbm_push_ctas<double>(batched);
    const int grid = (int)std::min<long long>((cells + 255) / 256, (long long)p->sms * bps);
    cudaError_t e = lbm_push_launch(p->dtype == ST_F32 ? 0 : 1, p->exact, !sv.single, batched, src, dst, sv.fl2, prm,
                                    grid, sv.stream ? sv.stream : p->stream);
    if (e != cudaSuccess) return fail(ST_ECUDA, "lbm launch: %s", cudaGetErrorString(e));
    ++p->launches;
    return ST_OK;
}

// one pass of the TMA gather form over the output planes [sv.za, sv.zb) of a
// (slab) buffer of sv.nzb planes (Z-slab schedule; the single-domain path
// encodes its maps once per run instead)
static int launch_lbm_tma_slab(st_plan* p, int mode, const void* src, void* dst, double omega, const SlabView& sv) {
    NvtxRange nvtx_(mode == LBM_COLLIDE ? "lbm collide pass" : mode == LBM_PULL ? "lbm pull pass" : "lbm stream pass");
    if (sv.zb <= sv.za) return ST_OK;
    const int dt = p->dtype == ST_F32 ? 0 : 1;
    int bx, by, halo;
    lbm_pull_tma_box(dt, p->nx, &bx, &by, &halo);
    CUtensorMap maps[2];
    for (int w = 0; w < 2; ++w) {
        int rc = encode_lbm(&maps[w], src, p->dtype, p->nx, p->ny, sv.nzb, bx + w * halo, by);
        if (rc) return rc;
    }
    LbmParams prm{};
    prm.nx = p->nx; prm.ny = p->ny; prm.nzb = sv.nzb; prm.zbase = sv.zbase; prm.nzg = p->nz;
    prm.za = sv.za; prm.zb = sv.zb;
    prm.omega = omega;
    if (p->dtype == ST_F32) lid_coeffs<float>(p->lid, prm.lidc);
    else lid_coeffs<double>(p->lid, prm.lidc);
    const size_t sb = lbm_pull_tma_stage_bytes(dt, p->nx);
    const int stages = p->opt_lbm_stages > 0 ? p->opt_lbm_stages : (dt == 0 ? 3 : 1);
    if ((size_t)stages * sb > p->smem_optin) return fail(ST_EUNSUPPORTED, "LBM pull ring of %d stages", stages);
    const int per_sm = std::max(1, std::min(2, (int)(p->smem_sm / ((size_t)stages * sb + 1024))));
    const int tcols = (p->nx + bx - 1) / bx;
    const long long tiles = (long long)tcols * ((p->ny + by - 1) / by) * (sv.zb - sv.za);
    long long cap = (long long)p->sms * per_sm;
    if (sv.grid_cap > 0) cap = std::min<long long>(cap, (long long)sv.grid_cap * per_sm);   // SMs left to NCCL
    int grid = (int)std::min<long long>(tiles, cap);
    if (grid > 1 && grid % tcols == 0) --grid;   // rotate the x-wall tiles over the CTAs (see runlbm_device)
    cudaError_t e = lbm_pull_tma_launch(dt, p->exact, mode, p->opt_pdl != 0, maps, src, dst, sv.fl2, prm, grid,
                                        stages, sv.stream ? sv.stream : p->stream);
    if (e != cudaSuccess) return fail(ST_ECUDA, "lbm TMA pass: %s", cudaGetErrorString(e));
    ++p->launches;
    return ST_OK;
}

static int check_shell(st_plan* p, const uint8_t* flags) {
    if (p->flags_checked == flags) return ST_OK;
    if (p->dist.mode == Dist::NCCL) { p->flags_checked = flags; return ST_OK; }  // caller-owned slab flags
    cudaError_t e = lbm_shell_check(flags, p->nx, p->ny, p->nz, p->d_count, p->stream);
    if (e != cudaSuccess) return fail(ST_ECUDA, "shell check: %s", cudaGetErrorString(e));
    CUDA_TRY(cudaMemcpyAsync(p->h_count, p->d_count, sizeof(int), cudaMemcpyDeviceToHost, p->stream));
    CUDA_TRY(cudaStreamSynchronize(p->stream));
    if (*p->h_count != 0)
        return fail(ST_EUNSUPPORTED, "%d shell cells are FLUID; the GPU path needs a non-FLUID shell", *p->h_count);
    p->flags_checked = flags;
    return ST_OK;
}

static int runlbm_device(st_plan* p, void* fsrc, void* fdst, double omega, int T, const uint8_t* flags) {
    const size_t n = 19 * (size_t)p->nx * p->ny * p->dist.nzb * esize(p->dtype);
    p->launches = 0;
    int rc = check_shell(p, flags);
    if (rc) return rc;
    if (T == 0) {
        CUDA_TRY(cudaMemcpyAsync(fdst, fsrc, n, cudaMemcpyDeviceToDevice, p->stream));
        return ST_OK;
    }
    // dim_T = 1: the fused push kernel (fastest measured on B200); dim_T >= 2:
    // the on-chip multi-level sweep lbm_35d (ST_OPT_LBM_KERNEL selects either)
    const bool push = lbm_use_push(p);
    // neighbour-flag prepass, every call (a reused flags pointer may hold new contents; ~1 pass over the flags)
    if (p->dist.mode != Dist::LOOPBACK) {
        const size_t cells = (size_t)p->nx * p->ny * p->dist.nzb;
        if (p->fl2_bytes < cells) {
            if (p->fl2) cudaFree(p->fl2);
            p->fl2 = nullptr; p->fl2_bytes = 0;
            if (cudaMalloc(&p->fl2, cells) != cudaSuccess) { cudaGetLastError(); return fail(ST_ENOMEM, "fl2"); }
            p->fl2_bytes = cells;
        }
        cudaError_t e = lbm_fl2(flags, p->fl2, p->nx, p->ny, p->dist.nzb, p->stream);
        if (e != cudaSuccess) return fail(ST_ECUDA, "fl2 prepass: %s", cudaGetErrorString(e));
    }
    // FP32 dim_T = 1 runs of T >= 4 steps: the gather form with TMA-fed passes
    // (measured on B200, 256^3 cavity: 34.1 vs 25.8 GLUPS for the push kernel; FP64
    // keeps push, 18.4 vs 16.7).  T + 1 passes.
    // Z slabs run the same T + 1 passes as depth-1 sweeps of the slab schedule
    // (one ghost plane per face exchanged before each pull / stream pass).
    int gk = p->opt_lbm_kernel;
    if (gk == 0 && push && p->dtype == ST_F32 && T >= 4 && ((size_t)p->nx * esize(p->dtype)) % 16 == 0)
        gk = 4;
    if (gk == 4 && p->dist.mode != Dist::SINGLE) {
        p->last_lbm_kernel = 400;
        rc = run_sweeps(p, std::vector<int>(T + 1, 1), fsrc, fdst, 19, flags,
                        [&](const void* a, void* b, int, const SlabView& sv) {
                            const int mode = sv.sweep == 0 ? LBM_COLLIDE : (sv.sweep == T ? LBM_STREAM : LBM_PULL);
                            return launch_lbm_tma_slab(p, mode, a, b, omega, sv);
                        });
        if (rc) return rc;
        CUDA_TRY(cudaGetLastError());
        return ST_OK;
    }
    if (gk == 3 || gk == 4) {   // gather form: C, T-1 pulls, S (single domain)
        if (p->dist.mode != Dist::SINGLE) return fail(ST_EUNSUPPORTED, "the plain gather-form LBM kernels are single-domain");
        LbmParams prm{};
        prm.nx = p->nx; prm.ny = p->ny; prm.nzb = p->nz; prm.zbase = 0; prm.nzg = p->nz;
        prm.za = 0; prm.zb = p->nz;
        prm.omega = omega;
        if (p->dtype == ST_F32) lid_coeffs<float>(p->lid, prm.lidc);
        else lid_coeffs<double>(p->lid, prm.lidc);
        const long long cells = (long long)p->nx * p->ny * p->nz;
        const int grid = (int)std::min<long long>((cells + 255) / 256, (long long)p->sms * 4);
        const int dt = p->dtype == ST_F32 ? 0 : 1;
        // TMA pulls (a10): 4D maps of both lattices, S-stage ring, CTAs per SM from shared memory
        const bool tma = gk == 4 && ((size_t)p->nx * esize(p->dtype)) % 16 == 0;
        p->last_lbm_kernel = tma ? 400 : 300;
        CUtensorMap map_src[2], map_dst[2];
        int tgrid = 0, stages = 0;
        if (tma) {
            int bx, by, halo;
            lbm_pull_tma_box(dt, p->nx, &bx, &by, &halo);
            for (int w = 0; w < 2 && !rc; ++w) {
                rc = encode_lbm(&map_src[w], fsrc, p->dtype, p->nx, p->ny, p->nz, bx + w * halo, by);
                if (!rc) rc = encode_lbm(&map_dst[w], fdst, p->dtype, p->nx, p->ny, p->nz, bx + w * halo, by);
            }
            if (rc) return rc;
            const size_t sb = lbm_pull_tma_stage_bytes(dt, p->nx);
            stages = p->opt_lbm_stages > 0 ? p->opt_lbm_stages : (dt == 0 ? 3 : 1);
            if ((size_t)stages * sb > p->smem_optin) return fail(ST_EUNSUPPORTED, "LBM pull ring of %d stages", stages);
            const int per_sm = std::max(1, std::min(2, (int)(p->smem_sm / ((size_t)stages * sb + 1024))));
            const long long tiles = (long long)((p->nx + bx - 1) / bx) * ((p->ny + by - 1) / by) * p->nz;
            tgrid = (int)std::min<long long>(tiles, (long long)p->sms * per_sm);
            // tiles are dealt round-robin: a grid that is a multiple of the tile
            // columns would give every CTA the same x position (and the CTAs holding
            // the x walls all the slow bounce-back cells); one CTA fewer rotates them
            const int tcols = (p->nx + bx - 1) / bx;
            if (tgrid > 1 && tgrid % tcols == 0) --tgrid;
        }
        // T + 1 passes; C in place when T is odd so the result lands in f_dst
        void* a = fsrc;
        void* b = fdst;
        auto pass = [&](int mode, void* from, void* to) -> int {
            NvtxRange nvtx_(mode == LBM_COLLIDE ? "lbm collide pass" : mode == LBM_PULL ? "lbm pull pass" : "lbm stream pass");
            cudaError_t e;
            if (tma)
                e = lbm_pull_tma_launch(dt, p->exact, mode, p->opt_pdl != 0, from == fsrc ? map_src : map_dst, from,
                                        to, p->fl2, prm, tgrid, stages, p->stream);
            else
                e = lbm_gather_launch(dt, p->exact, mode, from, to, p->fl2, prm, grid, p->stream);
            if (e != cudaSuccess) return fail(ST_ECUDA, "lbm gather launch: %s", cudaGetErrorString(e));
            ++p->launches;
            return ST_OK;
        };
        if (T % 2) { rc = pass(LBM_COLLIDE, a, a); }
        else { rc = pass(LBM_COLLIDE, a, b); std::swap(a, b); }
        for (int t = 1; t < T && !rc; ++t) { rc = pass(LBM_PULL, a, b); std::swap(a, b); }
        if (!rc) rc = pass(LBM_STREAM, a, b);
        if (rc) return rc;
        CUDA_TRY(cudaGetLastError());
        return ST_OK;
    }
    std::vector<int> ds = push ? std::vector<int>(T, 1) : sweep_depths(T, max_lbm_depth(p));
    p->last_lbm_kernel = push ? 100 : 200 + max_lbm_depth(p);
    rc = run_sweeps(p, ds, fsrc, fdst, 19, flags, [&](const void* a, void* b, int d, const SlabView& sv) {
        if (push) return launch_lbm(p, a, b, sv.flags, omega, sv);
        return launch_lbm35(p, a, b, d, omega, sv);
    });
    if (rc) return rc;
    CUDA_TRY(cudaGetLastError());
    return ST_OK;
}

extern "C" int lbm_d3q19_run(st_plan* p, void* fsrc, void* fdst, double omega, int T, const uint8_t* flags) {
    NvtxRange nvtx_("lbm_d3q19_run");
    if (!p) return fail(ST_EINVAL, "NULL plan");
    if (!fsrc || !fdst || !flags) return fail(ST_EINVAL, "NULL pointer");
    if (T < 0) return fail(ST_EINVAL, "T = %d < 0", T);
    if (!(omega >= 0.0 && omega < 2.0)) return fail(ST_EINVAL, "omega = %g not in [0, 2)", omega);
    const size_t cells = (size_t)p->nx * p->ny * p->dist.nzb;
    const size_t n = 19 * cells * esize(p->dtype);
    if (overlap(fsrc, fdst, n)) return fail(ST_EINVAL, "f_src and f_dst overlap");
    const int ks = ptr_kind(fsrc), kd = ptr_kind(fdst), kf = ptr_kind(flags);
    if (ks != kd || ks != kf) return fail(ST_EINVAL, "f_src, f_dst and flags must all be host or all device");
    if (ks == 1) {
        if ((reinterpret_cast<uintptr_t>(fsrc) | reinterpret_cast<uintptr_t>(fdst)) & 15)
            return fail(ST_EINVAL, "device lattices must be 16-byte aligned");
        return runlbm_device(p, fsrc, fdst, omega, T, flags);
    }
    int rc = ensure_hbuf(p, n);
    if (rc) return rc;
    if (p->hflags_bytes < cells) {
        if (p->hflags) cudaFree(p->hflags);
        p->hflags = nullptr; p->hflags_bytes = 0;
        if (cudaMalloc(&p->hflags, cells) != cudaSuccess) { cudaGetLastError(); return fail(ST_ENOMEM, "flags staging"); }
        p->hflags_bytes = cells;
    }
    CUDA_TRY(cudaMemcpyAsync(p->hbuf[0], fsrc, n, cudaMemcpyHostToDevice, p->stream));
    CUDA_TRY(cudaMemcpyAsync(p->hflags, flags, cells, cudaMemcpyHostToDevice, p->stream));
    p->flags_checked = nullptr;  // staging buffer content changes per call
    rc = runlbm_device(p, p->hbuf[0], p->hbuf[1], omega, T, p->hflags);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(fdst, p->hbuf[1], n, cudaMemcpyDeviceToHost, p->stream));
    CUDA_TRY(cudaStreamSynchronize(p->stream));
    return ST_OK;
}

// ----------------------------------------------------------------------------
// distribution (Z slabs)
// ----------------------------------------------------------------------------
#if ST_HAVE_NCCL
bool st35d::NcclApi::load() {
    if (h) return true;
    h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return false;
    getUniqueId = reinterpret_cast<decltype(getUniqueId)>(dlsym(h, "ncclGetUniqueId"));
    commInitRank = reinterpret_cast<decltype(commInitRank)>(dlsym(h, "ncclCommInitRank"));
    commInitRankConfig = reinterpret_cast<decltype(commInitRankConfig)>(dlsym(h, "ncclCommInitRankConfig"));
    commGetAsyncError = reinterpret_cast<decltype(commGetAsyncError)>(dlsym(h, "ncclCommGetAsyncError"));
    commDestroy = reinterpret_cast<decltype(commDestroy)>(dlsym(h, "ncclCommDestroy"));
    send = reinterpret_cast<decltype(send)>(dlsym(h, "ncclSend"));
    recv = reinterpret_cast<decltype(recv)>(dlsym(h, "ncclRecv"));
    groupStart = reinterpret_cast<decltype(groupStart)>(dlsym(h, "ncclGroupStart"));
    groupEnd = reinterpret_cast<decltype(groupEnd)>(dlsym(h, "ncclGroupEnd"));
    errorString = reinterpret_cast<decltype(errorString)>(dlsym(h, "ncclGetErrorString"));
    return getUniqueId && commInitRank && commDestroy && send && recv && groupStart && groupEnd && errorString;
}
st35d::NcclApi& st35d::nccl() {
    static NcclApi api;
    return api;
}
#endif

void st35d::Dist::destroy() {
    for (auto& s : slabs) {
        for (void*& b : s.buf) if (b) cudaFree(b);
        if (s.flags) cudaFree(s.flags);
        if (s.fl2) cudaFree(s.fl2);
    }
    slabs.clear();
    slab_cell_bytes = 0;
    slab_ncomp = 0;
#if ST_HAVE_NCCL
    if (nccl_comm) { nccl().commDestroy(nccl_comm); nccl_comm = nullptr; }
#endif
    if (comm) { cudaStreamSynchronize(comm); cudaStreamDestroy(comm); comm = nullptr; }
    if (ev_b) { cudaEventDestroy(ev_b); ev_b = nullptr; }
    if (ev_x) { cudaEventDestroy(ev_x); ev_x = nullptr; }
}

extern "C" int st_nccl_unique_id(void* out) {
    if (!out) return fail(ST_EINVAL, "NULL id buffer");
#if ST_HAVE_NCCL
    if (!nccl().load()) return fail(ST_ENCCL, "libnccl.so.2 not loadable (import torch first)");
    ncclUniqueId id;
    ncclResult_t r = nccl().getUniqueId(&id);
    if (r != ncclSuccess) return fail(ST_ENCCL, "ncclGetUniqueId: %s", nccl().errorString(r));
    memcpy(out, &id, sizeof id);
    return ST_OK;
#else
    return fail(ST_EUNSUPPORTED, "built without NCCL");
#endif
}

extern "C" int st_slab_range(int nz, int nranks, int rank, int* z0, int* nz_local) {
    if (nz < 1 || nranks < 1 || rank < 0 || rank >= nranks || nz < nranks) return fail(ST_EINVAL, "slab range");
    int a = 0, b = 0;
    slab_range(nz, nranks, rank, a, b);
    if (z0) *z0 = a;
    if (nz_local) *nz_local = b;
    return ST_OK;
}

extern "C" int st_slab_schedule(int nz, int nranks, int rank, int dim_T, int T, int overlap, st_slab_step* steps,
                                int max_steps) {
    if (nz < 1 || nranks < 1 || rank < 0 || rank >= nranks || nz < nranks || dim_T < 1 || T < 0)
        return fail(ST_EINVAL, "slab schedule arguments");
    if (nranks > 1 && nz / nranks < dim_T) return fail(ST_EINVAL, "slabs thinner than dim_T");
    int z0 = 0, nzl = 0;
    slab_range(nz, nranks, rank, z0, nzl);
    const std::vector<SlabStep> v = slab_schedule(sweep_depths(T, dim_T), dim_T, nzl, nz / nranks, overlap != 0);
    if (steps) {
        if (max_steps < (int)v.size()) return fail(ST_EINVAL, "schedule has %zu steps, room for %d", v.size(), max_steps);
        for (size_t i = 0; i < v.size(); ++i)
            steps[i] = st_slab_step{v[i].kind, v[i].sweep, v[i].depth, v[i].src, v[i].z_begin, v[i].z_end, v[i].async,
                                    v[i].grid_cap};
    }
    return (int)v.size();
}

extern "C" int st_plan_set_dist(st_plan* p, const void* uid, int rank, int nranks) {
    if (!p) return fail(ST_EINVAL, "NULL plan");
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(ST_EINVAL, "rank %d of %d", rank, nranks);
    CUDA_TRY(cudaStreamSynchronize(p->stream));
    if (nranks == 1 && !uid) { p->dist.init_single(p->nz); return ST_OK; }   // distribution off
    // (nranks == 1 with an id: a one-rank NCCL communicator running the full
    // distributed schedule -- the single-GPU test of the NCCL path)
    const int g = p->dimT;
    int z0 = 0, nzl = 0;
    slab_range(p->nz, nranks, rank, z0, nzl);
    if (p->nz / nranks < g) return fail(ST_EINVAL, "slabs of %d planes are thinner than dim_T %d", p->nz / nranks, g);
#if ST_HAVE_NCCL
    if (!uid) return fail(ST_EINVAL, "NULL NCCL unique id");
    if (!nccl().load()) return fail(ST_ENCCL, "libnccl.so.2 not loadable (import torch first)");
    p->dist.destroy();
    ncclUniqueId id;
    memcpy(&id, uid, sizeof id);
    ncclComm_t comm = nullptr;
    ncclResult_t r;
    if (nccl().commInitRankConfig) {
        // cap NCCL's CTAs so the exchange overlaps the interior sweep, which
        // leaves the same SMs free (run_sweeps grid cap)
        ncclConfig_t cfg = NCCL_CONFIG_INITIALIZER;
        cfg.blocking = 1;
        cfg.minCTAs = 1;
        cfg.maxCTAs = ST_NCCL_MAX_CTAS;
        r = nccl().commInitRankConfig(&comm, nranks, id, rank, &cfg);
        if (r != ncclSuccess) return fail(ST_ENCCL, "ncclCommInitRankConfig: %s", nccl().errorString(r));
    } else {
        r = nccl().commInitRank(&comm, nranks, id, rank);
        if (r != ncclSuccess) return fail(ST_ENCCL, "ncclCommInitRank: %s", nccl().errorString(r));
    }
    Dist& D = p->dist;
    p->geo7.clear();   // the kernel variant depends on the local slab
    D.mode = Dist::NCCL; D.nccl_comm = comm;
    D.nz = p->nz; D.P = nranks; D.rank = rank; D.g = g; D.z0 = z0; D.nzl = nzl; D.nzb = nzl + 2 * g;
    D.nranks = nranks;
    p->flags_checked = nullptr;
    return ST_OK;
#else
    (void)uid;
    return fail(ST_EUNSUPPORTED, "built without NCCL");
#endif
}

extern "C" int st_plan_set_loopback_slabs(st_plan* p, int nslabs) {
    if (!p) return fail(ST_EINVAL, "NULL plan");
    if (nslabs < 1) return fail(ST_EINVAL, "nslabs %d", nslabs);
    CUDA_TRY(cudaStreamSynchronize(p->stream));
    if (nslabs == 1) { p->dist.init_single(p->nz); return ST_OK; }
    const int g = p->dimT;
    if (p->nz / nslabs < g) return fail(ST_EINVAL, "slabs of %d planes are thinner than dim_T %d", p->nz / nslabs, g);
    Dist& D = p->dist;
    D.init_single(p->nz);      // caller buffers stay full grids in loopback mode
    D.mode = Dist::LOOPBACK; D.P = nslabs; D.g = g;
    D.slabs.resize(nslabs);
    for (int k = 0; k < nslabs; ++k) {
        slab_range(p->nz, nslabs, k, D.slabs[k].z0, D.slabs[k].nzl);
        D.slabs[k].nzb = D.slabs[k].nzl + 2 * g;
    }
    return ST_OK;
}
