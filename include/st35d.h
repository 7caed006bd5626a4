/*
 * st35d.h — C ABI of the B200 (sm_100a) 3.5D-blocked stencil sweeps.
 *
 * The operations are the two kernels of Nguyen et al., "3.5-D Blocking
 * Optimization for Stencil Computations on Modern CPUs and GPUs" (SC'10),
 * /root/reference/PAPER.md (cited P:<line>):
 *   - 7-point Jacobi stencil (§IV-A1, equation at; Jacobi two-grid
 *     sweep P:95; fixed boundary P:195),
 *   - D3Q19 lattice-Boltzmann collide+stream (§IV-B, steps 1-4 at P:125-132),
 * both executed by the 3.5D-blocked sweep of §V (2.5D spatial blocking of an
 * XY tile streamed along Z, plus dim_T time steps kept on chip,
 * P:183-255).  Blocking only reorders the computation, so the result
 * is that of T plain Jacobi sweeps.
 *
 * Memory layout: X fastest, then Y, then Z:
 *     idx(x,y,z) = (z*ny + y)*nx + x
 * LBM populations are SoA: f[i][z][y][x], i = 0..18, in the
 * velocity order of DESIGN.md (0 rest; 1..6 = +x,-x,+y,-y,+z,-z; 7..18 the
 * edge directions; opposite(i) = i+1 for odd i).  flags[z][y][x] is uint8:
 * 0 FLUID, 1 WALL (half-way bounce-back), 2 LID (moving wall, Ladd, rho_w=1).
 *
 * Ownership: the library never owns the grid buffers.  Pointers may be
 * DEVICE memory (the fast path: the call only enqueues kernels on the plan's
 * stream and returns) or HOST memory (pageable or pinned: the call copies to
 * plan-owned device scratch, runs, copies the result back and synchronises
 * before returning).  Host and device pointers may not be mixed in one call.
 *
 * Errors: every argument is checked before anything is launched; on error
 * nothing is written, the call returns a negative ST_E* code and
 * st_last_error() returns a thread-local message.  Device-side faults of an
 * asynchronous (device-pointer) run surface at the next call or at
 * st_plan_sync().  A plan is not thread-safe.
 */
#ifndef ST35D_H
#define ST35D_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct st_plan st_plan; /* opaque: owns streams, events, scratch, comm */

typedef enum { ST_F32 = 0, ST_F64 = 1 } st_dtype;

enum {
    ST_OK = 0,
    ST_EINVAL = -1,       /* bad argument (sizes, dim_T, T, omega, NULL pointer, aliasing) */
    ST_ENOMEM = -2,       /* device or host allocation failed                           */
    ST_ECUDA = -3,        /* CUDA runtime / driver error (incl. deferred device faults) */
    ST_ENCCL = -4,        /* NCCL error in the Z-slab ghost exchange                    */
    ST_EUNSUPPORTED = -5  /* valid request this build does not handle (see message)     */
};

enum { ST_FLUID = 0, ST_WALL = 1, ST_LID = 2 };

/* Maximum temporal blocking depth compiled into this build. */
#define ST_MAX_DIM_T 8

/*
 * st_plan_create — plan a sweep over an nx*ny*nz grid of `dtype` with
 * temporal blocking depth dim_T (number of time steps kept on chip per
 * sweep; eq. (3) P:225 says dim_T >= eta = ceil(gamma/Gamma)).
 * Requirements: nx, ny, nz >= 3; 1 <= dim_T <= ST_MAX_DIM_T;
 * nx*sizeof(dtype) a multiple of 16 bytes (TMA row-pitch rule).
 * The planner chooses the XY tile (eq. (1)/(4) analog for the on-chip bytes
 * of one SM) and the persistent grid that gives every CTA the same number of
 * tile-planes (flexible load balance).
 * nz is the GLOBAL number of planes even in distributed mode.
 * Returns NULL on error (st_last_error() says why).  Needs a CUDA device.
 */
st_plan* st_plan_create(int nx, int ny, int nz, st_dtype dtype, int dim_T);

/*
 * st7_run — out = A(T): T Jacobi sweeps of the 7-point stencil
 *     B = alpha*A + beta*(A[x-1]+A[x+1]+A[y-1]+A[y+1]+A[z-1]+A[z+1])
 * applied to every interior point; the shell x in {0,nx-1}, y in {0,ny-1},
 * z in {0,nz-1} is Dirichlet-fixed and copied.  alpha, beta are
 * rounded once to the plan dtype.  `in` and `out` are nx*ny*nz elements of
 * the plan dtype, must not overlap, and 16-byte aligned (device).  `in` is
 * SCRATCH: it is overwritten when more than one sweep runs (the two grids
 * ping-pong; no third grid is allocated).  T = 0 copies in to out.
 * In distributed mode (st_plan_set_dist) each rank passes its own slab
 * buffers of (nz_local + 2*g) planes, g = st_plan_ghost_planes(plan).
 */
int st7_run(st_plan* plan, const void* in, void* out, double alpha, double beta, int T);

/*
 * st27_run — out = A(T): T Jacobi sweeps of the 27-point stencil (P:119,
 * SURVEY §8(f) f1): "the edge points, corners and face neighbors are
 * multiplied by different constants",
 *     B = alpha*C + beta*(6 faces) + gamma*(12 edges) + delta*(8 corners)
 * over the 3x3x3 cube of every interior point; the shell is fixed as for
 * st7_run.  Summation order: DESIGN.md reading X24 (bit-identical to the
 * oracle with st_plan_set_bitexact(plan, 1), FMA-contracted otherwise).
 * Sweeps of depth min(dim_T, 4 FP32 / 2 FP64) are kept on chip (3.5D).  Same
 * buffers, ownership (`in` is scratch), pointer kinds (device: asynchronous
 * on the plan stream; host: staged and synchronous) and errors as st7_run.
 * Single process only: ST_EUNSUPPORTED after st_plan_set_dist.
 */
int st27_run(st_plan* plan, const void* in, void* out, double alpha, double beta, double gamma, double delta, int T);

/*
 * st13_run — out = A(T): T Jacobi sweeps of the radius-2 13-point star, the
 * general stencil radius R of §V ("the radius ... usually defined as
 * the Manhattan distance (e.g. k-point stencil)") with R = 2 (SURVEY §8(f)
 * f4; the paper runs only R = 1).  Reading X25:
 *     B = (alpha*C + beta*S1) + gamma*S2
 *     S1 = ((x-1 + x+1) + (y-1 + y+1)) + (z-1 + z+1), S2 likewise at distance 2
 * Reading X26: the fixed (Dirichlet) shell is 2 points thick on every face.
 * Sweeps of depth min(dim_T, 4 FP32 / 3 FP64) are kept on chip (3.5D, halo 2*dim_T,
 * lag R per level).  Requires every extent >= 5.  Same buffers, ownership
 * (`in` is scratch), pointer kinds and errors as st7_run; single process only.
 * Bit-identical to the oracle with st_plan_set_bitexact(plan, 1).
 */
int st13_run(st_plan* plan, const void* in, void* out, double alpha, double beta, double gamma, int T);

/*
 * lbm_d3q19_run — f_dst = state after T D3Q19 steps of f_src,
 * BGK single-relaxation collision with relaxation rate omega (0 <= omega < 2;
 * omega = 0 is pure streaming), push semantics: the stored state is
 * post-stream, pre-collision.  FLUID cells collide and propagate; a link into
 * a WALL cell bounces back (half-way); a link into a LID cell bounces back
 * with the Ladd correction -6*w_i*(e_i . u_lid) (rho_w = 1); non-FLUID cells
 * keep their 19 values.  f_src / f_dst are 19*nx*ny*nz elements (SoA), flags
 * nx*ny*nz bytes.  Every shell cell must be non-FLUID (else ST_EUNSUPPORTED).
 * f_src is SCRATCH (ping-pong partner).  T = 0 copies.
 */
int lbm_d3q19_run(st_plan* plan, void* f_src, void* f_dst, double omega, int T,
                  const uint8_t* flags);

/* st_destroy — free the plan (NULL-safe).  Waits for its stream first. */
void st_destroy(st_plan* plan);

/* Thread-local description of the last error ("" if none). */
const char* st_last_error(void);

/* Thread-local ST_E* code of the last error (ST_OK if none); lets callers of
 * st_plan_create (which returns NULL) see why. */
int st_last_status(void);

/* ---- optional setters / queries ------------------------------------------ */

/* Run on this cudaStream_t (default: a plan-owned non-blocking stream). */
int st_plan_set_stream(st_plan* plan, void* cuda_stream);

/* Moving-lid velocity for LID cells (default (0.05, 0, 0)). */
int st_plan_set_lbm_lid(st_plan* plan, double ux, double uy, double uz);

/* 1: bit-exact kernels (no FMA contraction, oracle operation order). */
int st_plan_set_bitexact(st_plan* plan, int on);

/* Kernel variant of st7_run (default ST_VARIANT_35D, the 3.5D sweep).
 * ST_VARIANT_NAIVE is the "no blocking" bar of the ablation ladder (PAPER.md
 * Fig. 5(b)): one Jacobi step per launch, one
 * thread per point, seven global loads per update, oracle operation order
 * (bit-identical to the oracle in either build).  Same contract as st7_run
 * (in is scratch, T = 0 copies); single-process plans only (a distributed
 * plan returns ST_EUNSUPPORTED at run time).  lbm_d3q19_run ignores it. */
enum { ST_VARIANT_35D = 0, ST_VARIANT_NAIVE = 1 };
int st_plan_set_variant(st_plan* plan, int variant);

/* Tuning and test selections (no environment variables are read).
 *   ST_OPT_LBM_BATCHED  -1 (default) auto: FP32 lattices above 2^24 cells use the
 *                       batched-flag push kernel; 0 / 1 force the per-direction /
 *                       batched kernel (FP64 always batches).
 *   ST_OPT_LBM_KERNEL   0 (default) auto: when the plan's LBM depth is 1, the
 *                       TMA gather form (4) for FP32 runs of T >= 4, else the
 *                       dim_T = 1 push kernel; at depth >= 2 the multi-level
 *                       on-chip kernel; 1 push (dim_T = 1 sweeps); 2 multi-level
 *                       kernel at the plan depth; 3 gather form (collide pass,
 *                       T-1 pull passes, stream pass; aligned stores; single
 *                       domain); 4 the same with every pass fed by TMA (boxes
 *                       shifted per population, S-stage shared-memory ring); on
 *                       Z slabs the T + 1 passes run as depth-1 sweeps of the
 *                       slab schedule (one ghost plane per face per pass).
 *   ST_OPT_LBM_STAGES   0 (default) auto; 1..8 stages of the TMA pull ring.
 *   ST_OPT_OVERLAP      1 (default): Z-slab ghost exchange overlapped with the
 *                       interior sweep on a side stream; 0 serialised.
 *   ST_OPT_PDL          1 (default): 7-point sweeps chained with programmatic
 *                       dependent launch; 0 plain launches.
 *   ST_OPT_ST7_VARIANT  0 (default) auto; else VY*1000 + threads per CTA
 *                       (+ 10000 * CTAs per SM) of a compiled 7-point kernel
 *                       variant: 4256, 4384, 2256, 2512, 22256; FP32 ablation
 *                       ladder: 1256 (one row per thread), 94256 (level by
 *                       level, no two-phase rounds).
 *   ST_OPT_ZCHUNK       0 (default); > 0: the 7-point sweep also restarts every
 *                       that many output planes of a tile, i.e. 3D blocks with
 *                       temporal blocking (the ablation ladder's 4D bar,
 *                       PAPER.md P:275-281).
 * Results do not depend on any option.  Unknown option or value: ST_EINVAL. */
enum { ST_OPT_LBM_BATCHED = 1, ST_OPT_LBM_KERNEL = 2, ST_OPT_OVERLAP = 3, ST_OPT_PDL = 4, ST_OPT_ST7_VARIANT = 5,
       ST_OPT_ZCHUNK = 6, ST_OPT_LBM_STAGES = 7 };
int st_plan_set_option(st_plan* plan, int option, int value);

/* st_plan_autotune_report — choose the 7-point sweep depth (the paper's
 * "framework that determines the various blocking parameters"; eqs.
 * (1)-(4) of §V-C) from a model seeded by measurement:
 *   gamma     = 2E/7 bytes per FP lane-op of the 7-point update;
 *   Gamma_eff = (bytes/s of a depth-1 sweep) / (FP lane-ops/s of the deepest
 *               sweep the plan tiles): what this device delivers to this
 *               kernel, issue limits included (the nominal-peak Gamma of
 *               eq. (3) is reported beside it);
 *   eta       = the smallest depth with dim_T / kappa(dim_T) >= gamma / Gamma_eff
 *               (eq. 3 with the planner's overestimation kappa, eq. 2)
 *               seeds the search: depths
 *               eta-1..eta+1 are timed and the search walks toward the faster
 *               neighbour until the best has timed neighbours on both sides;
 *   tile_side = eq. (4) at eta for three on-chip capacities C: one CTA's
 *               shared memory, the SM's shared memory + register file, and an
 *               8-CTA cluster's distributed shared memory.
 * Each timed depth runs T_probe Jacobi steps of st7_run on the caller's DEVICE
 * grids a and b (n^3 each, both clobbered), CUDA events on the plan stream;
 * results are identical for every depth.  The fastest depth becomes the
 * plan's st7_run sweep depth.  Synchronous.  Single-process plans only
 * (ST_EUNSUPPORTED otherwise: tune one rank and broadcast).  Returns the
 * chosen depth (>= 1) or < 0; rep (may be NULL) receives the report. */
typedef struct {
    int dim_T;                 /* chosen depth                                      */
    int eta;                   /* P:255 / eq. (3) with Gamma_eff and kappa          */
    int eta_nominal;           /* eq. (3) with the device's nominal peaks           */
    double gamma;              /* bytes per FP lane-op of the kernel                */
    double Gamma_nominal;      /* nominal HBM bytes/s / FP lane-ops/s               */
    double Gamma_eff;          /* measured (see above)                              */
    double bw_dim1;            /* measured algorithmic bytes/s at depth 1           */
    double fp_deep;            /* measured FP lane-ops/s at the deepest depth (ghost points incl.) */
    int tested[ST_MAX_DIM_T];  /* 1 where the depth was timed                       */
    float ms[ST_MAX_DIM_T];    /* time of T_probe steps per timed depth (0 untimed) */
    double capacity[3];        /* C (bytes): CTA smem, SM smem + RF, 8-CTA cluster  */
    int tile_side[3];          /* eq. (4) floor(sqrt(C / (E (2R+2) eta)))           */
    double kappa[3];           /* eq. (2) at that side and eta                      */
} st_autotune_report;
int st_plan_autotune_report(st_plan* plan, void* a, void* b, int T_probe, st_autotune_report* rep);

/* st_plan_autotune — the same search; eta_out (may be NULL) receives the
 * eq. (3) eta from the measured Gamma, ms_out (may be NULL, length >=
 * ST_MAX_DIM_T) the time per depth (0 for depths not timed). */
int st_plan_autotune(st_plan* plan, void* a, void* b, int T_probe, int* eta_out, float* ms_out);

/* Waits for the plan stream; returns ST_ECUDA for deferred device faults. */
int st_plan_sync(st_plan* plan);

/* Z-slab distribution (§8(e)): rank owns planes [z0, z0+nz_local) of the
 * global grid (remainder planes go one each to the first ranks).  The
 * 128-byte NCCL unique id comes from rank 0 (broadcast by the caller).
 * nranks == 1 with a NULL id switches distribution off; with an id it builds
 * a one-rank communicator that runs the distributed schedule (testing).
 * The communicator is created with ncclCommInitRankConfig, maxCTAs = 4 (the
 * exchange overlaps the interior sweep); asynchronous NCCL errors are polled
 * (ncclCommGetAsyncError) after every run and by st_plan_sync -> ST_ENCCL. */
int st_plan_set_dist(st_plan* plan, const void* nccl_unique_id, int rank, int nranks);

/* 128-byte NCCL unique id for st_plan_set_dist (call on rank 0, broadcast). */
int st_nccl_unique_id(void* out128);

/* Z-slab of `rank` among `nranks`: first global plane and plane count
 * (remainder planes one each to the first ranks).  Host-only. */
int st_slab_range(int nz, int nranks, int rank, int* z0, int* nz_local);

/* The Z-slab sweep schedule a rank of a distributed plan executes (host-only,
 * no device needed; st7_run / lbm_d3q19_run run exactly this list, SURVEY
 * §8(e)).  Buffer coordinates: plane L of a slab buffer is global plane
 * z0 - g + L, g = dim_T ghost planes per side, owned planes [g, g + nz_local).
 *   ST_STEP_EXCHANGE: send planes [g, g+depth) of buffer `src` to rank-1 and
 *     [g+nz_local-depth, g+nz_local) to rank+1; receive the neighbours' into
 *     [g-depth, g) and [g+nz_local, g+nz_local+depth) (a depth-d sweep
 *     needs d valid ghost planes per face).  async = 1: overlapped with the
 *     following ST_STEP_SWEEP steps, up to the next ST_STEP_WAIT.
 *   ST_STEP_SWEEP: `depth` Jacobi steps from buffer src into buffer 1-src for
 *     the output planes [z_begin, z_end) (grid_cap = 1: SMs left to NCCL).
 *   ST_STEP_WAIT: the sweep stream waits for the async exchange.
 *   ST_STEP_COPY: an even number of sweeps left the result in buffer 0 (`in`).
 * Buffer 0 is the caller's `in`, 1 its `out`.  overlap = 0 gives the
 * serialised schedule (ST_OPT_OVERLAP).  Returns the step count (steps may be
 * NULL to query it) or < 0. */
enum { ST_STEP_EXCHANGE = 0, ST_STEP_SWEEP = 1, ST_STEP_WAIT = 2, ST_STEP_COPY = 3 };
typedef struct {
    int kind, sweep, depth, src, z_begin, z_end, async, grid_cap;
} st_slab_step;
int st_slab_schedule(int nz, int nranks, int rank, int dim_T, int T, int overlap, st_slab_step* steps, int max_steps);

/* Loopback distribution on one device (testing): P virtual slabs, ghosts
 * copied with cudaMemcpyAsync instead of NCCL; result identical to P = 1. */
int st_plan_set_loopback_slabs(st_plan* plan, int nslabs);

/* g = dim_T ghost planes per side of each slab in distributed mode (R = 1). */
int st_plan_ghost_planes(const st_plan* plan);

/* Local slab extent of this rank: first global plane and plane count. */
int st_plan_local_slab(const st_plan* plan, int* z0, int* nz_local);

/* Planner decisions, for logging/bench: tile TX x TY (loaded, incl. halo),
 * output tile W_x x W_y, number of XY tiles, persistent CTAs, kernel variant. */
typedef struct {
    int tile_x, tile_y;     /* loaded XY sub-plane (dim_X, dim_Y of eq. (1))   */
    int out_x, out_y;       /* written region per tile (dim - 2*R*dim_T) */
    int tiles_x, tiles_y;   /* XY tiles covering the plane                      */
    int ctas;               /* persistent CTAs launched per sweep               */
    int threads;            /* threads per CTA                                  */
    int smem_bytes;         /* dynamic shared memory per CTA                    */
    double kappa;           /* eq. (2) analog: computed / useful points         */
    int kernel;             /* internal variant id; LBM (after a run: the kernel
                               it used): 100 push, 200+d multi-level of depth d,
                               300 gather form, 400 gather form with TMA pulls  */
    int dim_t_sweep;        /* deepest sweep actually run (<= dim_T, see above)  */
    int ring;               /* TMA plane-ring slots (ring-2 planes in flight)    */
} st_plan_info;
int st_plan_get_info(const st_plan* plan, int lbm, st_plan_info* info);

/* Number of kernel launches the last run enqueued (bench accounting). */
int st_plan_last_launches(const st_plan* plan);

/*
 * Blocking-parameter model of §V-C (host-only, no device needed):
 *   eq. (1)  E*(2R+2)*dim_T*dim_X*dim_Y <= C
 *   eq. (2)  kappa = ((1-2R dim_T/dim_X)(1-2R dim_T/dim_Y))^-1
 *   eq. (3)  dim_T >= eta = ceil(gamma/Gamma)
 *   eq. (4)  dim_X = dim_Y = floor(sqrt(C/(E*(2R+2)*eta)))
 * st_blocking_model fills eta, the eq. (4) real bound (before floor) and
 * kappa for the given dim (dim <= 0: use the eq. (4) floor).
 */
typedef struct {
    int eta;
    double dim_bound;   /* sqrt(C/(E(2R+2)eta)) */
    int dim;            /* tile side used for kappa */
    double kappa;
} st_blocking;
int st_blocking_model(double C_bytes, double E_bytes, int R, double gamma, double Gamma,
                      int dim_T, int dim, st_blocking* out);

/* Paper's Fig. 3 buffer schedule (R, dim_T): at round r (0-based), level t'
 * (0..dim_T) handles plane z = r - 2*R*t' in buffer slot
 * z mod (2R+2); returns the step number S (1-based, chronological as in
 * Fig. 3(a)) or 0 if level t' is idle in that round. */
int st_fig3_step(int R, int dim_T, int round, int level, int* z, int* slot);

#ifdef __cplusplus
}
#endif
#endif /* ST35D_H */
