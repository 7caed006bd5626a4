/*
 * oracle.c — plain, slow, obviously-correct CPU oracle for the two kernels of
 *   Nguyen, Satish, Chhugani, Kim, Dubey, "3.5-D Blocking Optimization for
 *   Stencil Computations on Modern CPUs and GPUs", SC'10
 *   (/root/reference/PAPER.md, cited P:<line>).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this code.  It
 * shares no code, header, table or helper with the CUDA path
 * (paper_conf_sc_nguyensckd10_b200/csrc) and never includes it.
 *
 * 3.5D blocking only reorders the computation ("performing dim_T time steps
 * only requires grid elements to be read and written once"), so the
 * oracle is the plain definition: T naive Jacobi sweeps of
 *   - the 7-point stencil, P:111 (eq. in §IV-A1),
 *   - the radius-2 13-point star (general R of §V; readings X25/X26),
 *   - the 27-point stencil, and
 *   - the D3Q19 lattice-Boltzmann step, P:125-132 (§IV-B, push form).
 * Readings of silent/ambiguous points are DESIGN.md X1..X21.
 *
 * Arithmetic is in the plan dtype (the paper fixes SP and DP),
 * compiled with -O2 -ffp-contract=off and no fast-math, so every product and
 * sum is rounded separately in the order written here (X2, X18).  The z loop
 * may run under OpenMP; each output point is computed by exactly one
 * iteration from the previous time level only, so the result is bit-identical
 * to the serial loop.
 *
 * Pins (tests/test_oracle_*.py): constant fixed point, Dirichlet eigenmode
 * closed form, impulse response (tests/golden/), brute-force recursion on 8^3,
 * mirror/transpose symmetries, T-split; D3Q19 lattice identities, equilibrium
 * moments, periodic mass/momentum conservation, cavity mass conservation,
 * uniform-equilibrium fixed point, omega=0 pure streaming == np.roll,
 * independent pull-form brute force, shear-wave decay.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define IDX(x, y, z) (((size_t)(z) * (size_t)ny + (size_t)(y)) * (size_t)nx + (size_t)(x))

/* ------------------------------------------------------------------------ */
/* 7-point stencil:                                                  */
/*   B(t+1) = alpha*A(t) + beta*(A[x-1]+A[x+1]+A[y-1]+A[y+1]+A[z-1]+A[z+1])  */
/* Jacobi two-grid sweep with swap.  Shell fixed (X1: "z0 (boundary   */
/* condition) does not change with time", applied to all 6 faces).    */
/* Summation order (X2): ((x-+x+) + (y-+y+)) + (z-+z+), two separate          */
/* products and one add ("2 multiplications, 6 additions").           */
/* ------------------------------------------------------------------------ */
#define DEFINE_ST7(TYPE, SUFFIX)                                                      \
int oracle_st7_##SUFFIX(const TYPE* A0, TYPE* out, long nx, long ny, long nz,         \
                        double alpha_d, double beta_d, int T)                         \
{                                                                                     \
    if (nx < 1 || ny < 1 || nz < 1 || T < 0) return -1;                               \
    const size_t n = (size_t)nx * ny * nz;                                            \
    const TYPE alpha = (TYPE)alpha_d, beta = (TYPE)beta_d; /* X19 */                  \
    TYPE* a = (TYPE*)malloc(n * sizeof(TYPE));                                        \
    TYPE* b = (TYPE*)malloc(n * sizeof(TYPE));                                        \
    if (!a || !b) { free(a); free(b); return -2; }                                    \
    memcpy(a, A0, n * sizeof(TYPE));                                                  \
    memcpy(b, A0, n * sizeof(TYPE));          /* both grids carry the shell */        \
    for (int t = 0; t < T; ++t) {                                                     \
        _Pragma("omp parallel for schedule(static)")                                  \
        for (long z = 1; z < nz - 1; ++z)                                             \
            for (long y = 1; y < ny - 1; ++y)                                         \
                for (long x = 1; x < nx - 1; ++x) {                                   \
                    TYPE sx = a[IDX(x - 1, y, z)] + a[IDX(x + 1, y, z)];              \
                    TYPE sy = a[IDX(x, y - 1, z)] + a[IDX(x, y + 1, z)];              \
                    TYPE sz = a[IDX(x, y, z - 1)] + a[IDX(x, y, z + 1)];              \
                    TYPE s = (sx + sy) + sz;                                          \
                    TYPE p = alpha * a[IDX(x, y, z)];                                 \
                    TYPE q = beta * s;                                                \
                    b[IDX(x, y, z)] = p + q;                                          \
                }                                                                     \
        TYPE* tmp = a; a = b; b = tmp;           /* swap roles */              \
    }                                                                                 \
    memcpy(out, a, n * sizeof(TYPE));                                                 \
    free(a); free(b);                                                                 \
    return 0;                                                                         \
}
DEFINE_ST7(float, f32)
DEFINE_ST7(double, f64)

/* ------------------------------------------------------------------------ */
/* Radius-2 star stencil, 13 points (the paper's general   */
/* radius R of §V, "the radius (in units) of extent of the stencil,    */
/* usually defined as the Manhattan distance (e.g. k-point stencil)", used   */
/* in every blocking formula of §V, but only run with R = 1,      */
/* P:259).  Reading X25 (the paper gives no R = 2 kernel):                    */
/*   B = (alpha*C + beta*S1) + gamma*S2                                      */
/*   S1 = ((x-1 + x+1) + (y-1 + y+1)) + (z-1 + z+1)   (the 7-point order X2) */
/*   S2 = ((x-2 + x+2) + (y-2 + y+2)) + (z-2 + z+2)                          */
/* three separately rounded products, 10 + 2 additions.  Reading X26: the    */
/* fixed (Dirichlet) shell is R = 2 points thick on every face (the points   */
/* whose stencil would leave the grid never change, as z0 in P:195).         */
/* With alpha = 1 - 7.5 nu, beta = 4 nu / 3, gamma = -nu / 12 this is the    */
/* explicit heat step with the 4th-order Laplacian (exact on polynomials of  */
/* degree <= 5, the pin of tests/test_oracle_st13.py).                       */
/* ------------------------------------------------------------------------ */
#define DEFINE_ST13(TYPE, SUFFIX)                                                     \
int oracle_st13_##SUFFIX(const TYPE* A0, TYPE* out, long nx, long ny, long nz,        \
                         double alpha_d, double beta_d, double gamma_d, int T)        \
{                                                                                     \
    if (nx < 1 || ny < 1 || nz < 1 || T < 0) return -1;                               \
    const size_t n = (size_t)nx * ny * nz;                                            \
    const TYPE alpha = (TYPE)alpha_d, beta = (TYPE)beta_d, gamma = (TYPE)gamma_d;     \
    TYPE* a = (TYPE*)malloc(n * sizeof(TYPE));                                        \
    TYPE* b = (TYPE*)malloc(n * sizeof(TYPE));                                        \
    if (!a || !b) { free(a); free(b); return -2; }                                    \
    memcpy(a, A0, n * sizeof(TYPE));                                                  \
    memcpy(b, A0, n * sizeof(TYPE));          /* both grids carry the shell */        \
    for (int t = 0; t < T; ++t) {                                                     \
        _Pragma("omp parallel for schedule(static)")                                  \
        for (long z = 2; z < nz - 2; ++z)                                             \
            for (long y = 2; y < ny - 2; ++y)                                         \
                for (long x = 2; x < nx - 2; ++x) {                                   \
                    TYPE sx1 = a[IDX(x - 1, y, z)] + a[IDX(x + 1, y, z)];             \
                    TYPE sy1 = a[IDX(x, y - 1, z)] + a[IDX(x, y + 1, z)];             \
                    TYPE sz1 = a[IDX(x, y, z - 1)] + a[IDX(x, y, z + 1)];             \
                    TYPE sx2 = a[IDX(x - 2, y, z)] + a[IDX(x + 2, y, z)];             \
                    TYPE sy2 = a[IDX(x, y - 2, z)] + a[IDX(x, y + 2, z)];             \
                    TYPE sz2 = a[IDX(x, y, z - 2)] + a[IDX(x, y, z + 2)];             \
                    TYPE s1 = (sx1 + sy1) + sz1;                                      \
                    TYPE s2 = (sx2 + sy2) + sz2;                                      \
                    TYPE p = alpha * a[IDX(x, y, z)];                                 \
                    TYPE q = beta * s1;                                               \
                    TYPE r = gamma * s2;                                              \
                    b[IDX(x, y, z)] = (p + q) + r;                                    \
                }                                                                     \
        TYPE* tmp = a; a = b; b = tmp;           /* swap roles */              \
    }                                                                                 \
    memcpy(out, a, n * sizeof(TYPE));                                                 \
    free(a); free(b);                                                                 \
    return 0;                                                                         \
}
DEFINE_ST13(float, f32)
DEFINE_ST13(double, f64)

/* ------------------------------------------------------------------------ */
/* 27-point stencil: the 3x3x3 cube around the      */
/* centre; "the edge points, corners and face neighbors are multiplied by    */
/* different constants", "4 multiplies, 26 adds":                            */
/*   B = alpha*C + beta*F + gamma*E + delta*K                                */
/* C centre, F the 6 face neighbours (one offset non-zero), E the 12 edge    */
/* points (two offsets non-zero), K the 8 corners (three non-zero).          */
/* Same Jacobi sweep / swap and fixed shell (X1) as the 7-point.      */
/* Summation order (reading X24; the paper gives none): with, for plane      */
/* z+dz,  v(dx) = a[dx,-1,dz] + a[dx,+1,dz]   (the y pair of column dx),     */
/*        h     = a[-1,0,dz]  + a[+1,0,dz]    (the x pair),                  */
/*        f(dz) = h + v(0)       (the 4 in-plane face points of plane dz),   */
/*        e(dz) = v(-1) + v(+1)  (the 4 in-plane corner points of plane dz), */
/*   F = f(0) + (a[0,0,-1] + a[0,0,+1])                                      */
/*   E = e(0) + (f(-1) + f(+1))                                              */
/*   K = e(-1) + e(+1)                                                       */
/*   B = ((alpha*C + beta*F) + gamma*E) + delta*K                            */
/* Each of the 26 neighbours enters exactly once: 4+2 / 4+4+4 / 4+4, and    */
/* there are 26 additions (F 5, E 11, K 7, final 3) and 4 products, as      */
/* P:119 counts.  F has the 7-point order of X2; every pair is symmetric,   */
/* so x, y and z mirrors are bit-exact.                                      */
/* ------------------------------------------------------------------------ */
#define DEFINE_ST27(TYPE, SUFFIX)                                                     \
static TYPE st27_f_##SUFFIX(const TYPE* a, long nx, long ny, long x, long y, long z)  \
{                                                                                     \
    TYPE h = a[IDX(x - 1, y, z)] + a[IDX(x + 1, y, z)];                               \
    TYPE v = a[IDX(x, y - 1, z)] + a[IDX(x, y + 1, z)];                               \
    return h + v;                                                                     \
}                                                                                     \
static TYPE st27_e_##SUFFIX(const TYPE* a, long nx, long ny, long x, long y, long z)  \
{                                                                                     \
    TYPE vm = a[IDX(x - 1, y - 1, z)] + a[IDX(x - 1, y + 1, z)];                      \
    TYPE vp = a[IDX(x + 1, y - 1, z)] + a[IDX(x + 1, y + 1, z)];                      \
    return vm + vp;                                                                   \
}                                                                                     \
int oracle_st27_##SUFFIX(const TYPE* A0, TYPE* out, long nx, long ny, long nz,        \
                         double alpha_d, double beta_d, double gamma_d,               \
                         double delta_d, int T)                                       \
{                                                                                     \
    if (nx < 1 || ny < 1 || nz < 1 || T < 0) return -1;                               \
    const size_t n = (size_t)nx * ny * nz;                                            \
    const TYPE alpha = (TYPE)alpha_d, beta = (TYPE)beta_d;   /* X19 */                \
    const TYPE gamma = (TYPE)gamma_d, delta = (TYPE)delta_d;                          \
    TYPE* a = (TYPE*)malloc(n * sizeof(TYPE));                                        \
    TYPE* b = (TYPE*)malloc(n * sizeof(TYPE));                                        \
    if (!a || !b) { free(a); free(b); return -2; }                                    \
    memcpy(a, A0, n * sizeof(TYPE));                                                  \
    memcpy(b, A0, n * sizeof(TYPE));                                                  \
    for (int t = 0; t < T; ++t) {                                                     \
        _Pragma("omp parallel for schedule(static)")                                  \
        for (long z = 1; z < nz - 1; ++z)                                             \
            for (long y = 1; y < ny - 1; ++y)                                         \
                for (long x = 1; x < nx - 1; ++x) {                                   \
                    TYPE zc = a[IDX(x, y, z - 1)] + a[IDX(x, y, z + 1)];              \
                    TYPE F = st27_f_##SUFFIX(a, nx, ny, x, y, z) + zc;                \
                    TYPE E = st27_e_##SUFFIX(a, nx, ny, x, y, z)                      \
                             + (st27_f_##SUFFIX(a, nx, ny, x, y, z - 1)               \
                                + st27_f_##SUFFIX(a, nx, ny, x, y, z + 1));           \
                    TYPE K = st27_e_##SUFFIX(a, nx, ny, x, y, z - 1)                  \
                             + st27_e_##SUFFIX(a, nx, ny, x, y, z + 1);               \
                    TYPE p = alpha * a[IDX(x, y, z)];                                 \
                    TYPE q = beta * F;                                                \
                    TYPE r = gamma * E;                                               \
                    TYPE s = delta * K;                                               \
                    b[IDX(x, y, z)] = ((p + q) + r) + s;                              \
                }                                                                     \
        TYPE* tmp = a; a = b; b = tmp;                                                \
    }                                                                                 \
    memcpy(out, a, n * sizeof(TYPE));                                                 \
    free(a); free(b);                                                                 \
    return 0;                                                                         \
}
DEFINE_ST27(float, f32)
DEFINE_ST27(double, f64)

/* ------------------------------------------------------------------------ */
/* D3Q19 lattice Boltzmann, push form (X13):                     */
/*   1. read the 19 values of the cell and its flag           */
/*   2. compute new values: BGK collision (X9)                               */
/*   3. propagate the 19 new values to the 18 neighbours and the local site  */
/*   4. swap source and destination                                  */
/* Stored state = post-stream, pre-collision.                                */
/* Velocity set, weights and boundary rules: DESIGN.md X10, X14.             */
/* ------------------------------------------------------------------------ */
static const int EX[19] = {0, 1, -1, 0, 0, 0, 0, 1, -1, 1, -1, 1, -1, 1, -1, 0, 0, 0, 0};
static const int EY[19] = {0, 0, 0, 1, -1, 0, 0, 1, -1, -1, 1, 0, 0, 0, 0, 1, -1, 1, -1};
static const int EZ[19] = {0, 0, 0, 0, 0, 1, -1, 0, 0, 0, 0, 1, -1, -1, 1, 1, -1, -1, 1};
static const int WDEN[19] = {3, 18, 18, 18, 18, 18, 18, 36, 36, 36, 36, 36, 36, 36, 36, 36, 36, 36, 36};

static int opp_of(int i) { return i == 0 ? 0 : ((i & 1) ? i + 1 : i - 1); }

enum { O_FLUID = 0, O_WALL = 1, O_LID = 2 };

/* tables exported for the lattice-identity pins (P6) */
void oracle_d3q19_tables(int* ex, int* ey, int* ez, int* wden, int* opp)
{
    for (int i = 0; i < 19; ++i) {
        ex[i] = EX[i]; ey[i] = EY[i]; ez[i] = EZ[i]; wden[i] = WDEN[i]; opp[i] = opp_of(i);
    }
}

/* BGK collision of one cell, in the order DESIGN.md X20 fixes.               */
#define DEFINE_COLLIDE(TYPE, SUFFIX)                                                  \
static void collide_##SUFFIX(const TYPE f[19], TYPE omega, TYPE fs[19], TYPE* rho_o)  \
{                                                                                     \
    TYPE rho = 0, jx = 0, jy = 0, jz = 0;                                             \
    for (int i = 0; i < 19; ++i) rho = rho + f[i];                                    \
    for (int i = 0; i < 19; ++i) {                                                    \
        if (EX[i]) jx = jx + (TYPE)EX[i] * f[i];                                      \
        if (EY[i]) jy = jy + (TYPE)EY[i] * f[i];                                      \
        if (EZ[i]) jz = jz + (TYPE)EZ[i] * f[i];                                      \
    }                                                                                 \
    TYPE ux = jx / rho, uy = jy / rho, uz = jz / rho;                                 \
    TYPE usq = ux * ux + uy * uy;                                                     \
    usq = usq + uz * uz;                                                              \
    TYPE usq15 = (TYPE)1.5 * usq;                                                     \
    for (int i = 0; i < 19; ++i) {                                                    \
        TYPE eu = 0;                                                                  \
        int first = 1;                                                                \
        if (EX[i]) { eu = (TYPE)EX[i] * ux; first = 0; }                              \
        if (EY[i]) { TYPE v = (TYPE)EY[i] * uy; eu = first ? v : eu + v; first = 0; } \
        if (EZ[i]) { TYPE v = (TYPE)EZ[i] * uz; eu = first ? v : eu + v; first = 0; } \
        TYPE w = (TYPE)1 / (TYPE)WDEN[i];                                             \
        TYPE wr = w * rho;                                                            \
        TYPE a = (TYPE)1 + (TYPE)3 * eu;                                              \
        TYPE c = ((TYPE)4.5 * eu) * eu;                                               \
        TYPE g = (a + c) - usq15;                                                     \
        TYPE feq = wr * g;                                                            \
        fs[i] = f[i] - omega * (f[i] - feq);                                          \
    }                                                                                 \
    *rho_o = rho;                                                                     \
}                                                                                     \
/* equilibrium alone, exported for the moment pins (P7) */                           \
void oracle_feq_##SUFFIX(double rho_d, double ux_d, double uy_d, double uz_d,         \
                         TYPE out[19])                                                \
{                                                                                     \
    TYPE rho = (TYPE)rho_d, ux = (TYPE)ux_d, uy = (TYPE)uy_d, uz = (TYPE)uz_d;        \
    TYPE usq = ux * ux + uy * uy;                                                     \
    usq = usq + uz * uz;                                                              \
    TYPE usq15 = (TYPE)1.5 * usq;                                                     \
    for (int i = 0; i < 19; ++i) {                                                    \
        TYPE eu = 0;                                                                  \
        int first = 1;                                                                \
        if (EX[i]) { eu = (TYPE)EX[i] * ux; first = 0; }                              \
        if (EY[i]) { TYPE v = (TYPE)EY[i] * uy; eu = first ? v : eu + v; first = 0; } \
        if (EZ[i]) { TYPE v = (TYPE)EZ[i] * uz; eu = first ? v : eu + v; first = 0; } \
        TYPE w = (TYPE)1 / (TYPE)WDEN[i];                                             \
        TYPE a = (TYPE)1 + (TYPE)3 * eu;                                              \
        TYPE c = ((TYPE)4.5 * eu) * eu;                                               \
        out[i] = (w * rho) * ((a + c) - usq15);                                       \
    }                                                                                 \
}
DEFINE_COLLIDE(float, f32)
DEFINE_COLLIDE(double, f64)

/*
 * One run of T push steps.  f_src/f_dst are [19][nz][ny][nx] (SoA);
 * flags [nz][ny][nx] uint8 (0 FLUID, 1 WALL, 2 LID).  periodic != 0 wraps the
 * neighbour index (oracle-only; used by the conservation pins); otherwise a
 * target outside the lattice is treated as WALL.
 * Lid rule (Ladd moving wall, rho_w = 1, X10/X14):
 *   f_dst[opp(i)][x] = f*_i(x) - (6*w_i) * (e_i . u_lid)
 * with e_i . u_lid summed over the non-zero components in x, y, z order.
 * Non-FLUID cells copy their 19 values through unchanged.
 */
#define DEFINE_LBM(TYPE, SUFFIX)                                                      \
int oracle_lbm_##SUFFIX(const TYPE* f0, TYPE* out, const uint8_t* flags,              \
                        long nx, long ny, long nz, double omega_d, int T,             \
                        double ulx, double uly, double ulz, int periodic)             \
{                                                                                     \
    if (nx < 1 || ny < 1 || nz < 1 || T < 0) return -1;                               \
    const size_t nc = (size_t)nx * ny * nz;                                           \
    const TYPE omega = (TYPE)omega_d;                                                 \
    const TYPE uw[3] = {(TYPE)ulx, (TYPE)uly, (TYPE)ulz};                             \
    TYPE lidc[19];                                                                    \
    for (int i = 0; i < 19; ++i) {                                                    \
        TYPE eu = 0; int first = 1;                                                   \
        if (EX[i]) { eu = (TYPE)EX[i] * uw[0]; first = 0; }                           \
        if (EY[i]) { TYPE v = (TYPE)EY[i] * uw[1]; eu = first ? v : eu + v; first = 0; } \
        if (EZ[i]) { TYPE v = (TYPE)EZ[i] * uw[2]; eu = first ? v : eu + v; first = 0; } \
        TYPE w = (TYPE)1 / (TYPE)WDEN[i];                                             \
        lidc[i] = ((TYPE)6 * w) * eu;                                                 \
    }                                                                                 \
    TYPE* a = (TYPE*)malloc(19 * nc * sizeof(TYPE));                                  \
    TYPE* b = (TYPE*)malloc(19 * nc * sizeof(TYPE));                                  \
    if (!a || !b) { free(a); free(b); return -2; }                                    \
    memcpy(a, f0, 19 * nc * sizeof(TYPE));                                            \
    for (int t = 0; t < T; ++t) {                                                     \
        _Pragma("omp parallel for schedule(static)")                                  \
        for (long z = 0; z < nz; ++z)                                                 \
            for (long y = 0; y < ny; ++y)                                             \
                for (long x = 0; x < nx; ++x) {                                       \
                    size_t c = IDX(x, y, z);                                          \
                    if (flags[c] != O_FLUID) {                                        \
                        for (int i = 0; i < 19; ++i) b[i * nc + c] = a[i * nc + c];   \
                        continue;                                                     \
                    }                                                                 \
                    TYPE f[19], fs[19], rho;                                          \
                    for (int i = 0; i < 19; ++i) f[i] = a[i * nc + c];                \
                    collide_##SUFFIX(f, omega, fs, &rho);                             \
                    for (int i = 0; i < 19; ++i) {                                    \
                        long tx = x + EX[i], ty = y + EY[i], tz = z + EZ[i];          \
                        int tflag;                                                    \
                        if (periodic) {                                               \
                            tx = (tx + nx) % nx; ty = (ty + ny) % ny; tz = (tz + nz) % nz; \
                            tflag = flags[IDX(tx, ty, tz)];                           \
                        } else if (tx < 0 || ty < 0 || tz < 0 ||                      \
                                   tx >= nx || ty >= ny || tz >= nz) {                \
                            tflag = O_WALL;                                           \
                        } else {                                                      \
                            tflag = flags[IDX(tx, ty, tz)];                           \
                        }                                                             \
                        if (tflag == O_FLUID)                                         \
                            b[i * nc + IDX(tx, ty, tz)] = fs[i];                      \
                        else if (tflag == O_WALL)                                     \
                            b[opp_of(i) * nc + c] = fs[i];                            \
                        else                                                          \
                            b[opp_of(i) * nc + c] = fs[i] - lidc[i];                  \
                    }                                                                 \
                }                                                                     \
        TYPE* tmp = a; a = b; b = tmp;                                                \
    }                                                                                 \
    memcpy(out, a, 19 * nc * sizeof(TYPE));                                           \
    free(a); free(b);                                                                 \
    return 0;                                                                         \
}
DEFINE_LBM(float, f32)
DEFINE_LBM(double, f64)

int oracle_num_threads(void)
{
#ifdef _OPENMP
    extern int omp_get_max_threads(void);
    return omp_get_max_threads();
#else
    return 1;
#endif
}
