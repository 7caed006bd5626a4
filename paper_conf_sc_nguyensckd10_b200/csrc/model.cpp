// model.cpp — host-only pieces of the C ABI that need no device:
//   * the blocking-parameter model of PAPER.md §V-C, eqs. (1)-(4)
//   * the paper's Fig. 3 buffer schedule
#include <cmath>
#include "../../include/st35d.h"

extern "C" int st_blocking_model(double C_bytes, double E_bytes, int R, double gamma, double Gamma, int dim_T,
                                 int dim, st_blocking* out) {
    if (!out || C_bytes <= 0 || E_bytes <= 0 || R < 1 || gamma <= 0 || Gamma <= 0) return ST_EINVAL;
    // eq. (3): dim_T >= eta = ceil(gamma / Gamma)
    out->eta = (int)std::ceil(gamma / Gamma - 1e-12);
    if (out->eta < 1) out->eta = 1;
    const int dt = dim_T > 0 ? dim_T : out->eta;
    // eq. (4): dim_X = dim_Y = floor(sqrt(C / (E (2R+2) eta)))  (eq. (1) at equality)
    out->dim_bound = std::sqrt(C_bytes / (E_bytes * (2.0 * R + 2.0) * dt));
    out->dim = dim > 0 ? dim : (int)std::floor(out->dim_bound);
    // eq. (2): kappa = ((1 - 2R dim_T/dim_X)(1 - 2R dim_T/dim_Y))^-1
    const double f = 1.0 - 2.0 * R * dt / (double)out->dim;
    out->kappa = f > 0 ? 1.0 / (f * f) : INFINITY;
    return ST_OK;
}

// Fig. 3(a) (R = 1, dim_T = 3 in the paper): round r loads plane r at t' = 0
// and computes plane z = r - 2R t' at level t' (z_s = z + 2R(dim_T - t'')
// for the plane stored at round z + 2R dim_T).  Level t' >= 1 is busy only
// when z >= R (z0 is boundary).  Steps are numbered chronologically,
// levels in increasing order within a round (S8, S9, S10 at round 5).
extern "C" int st_fig3_step(int R, int dim_T, int round, int level, int* z_out, int* slot_out) {
    if (R < 1 || dim_T < 1 || round < 0 || level < 0 || level > dim_T) return ST_EINVAL;
    auto active = [&](int r, int t) {
        const int z = r - 2 * R * t;
        return t == 0 ? z >= 0 : z >= R;
    };
    if (!active(round, level)) return 0;
    int step = 0;
    for (int r = 0; r <= round; ++r)
        for (int t = 0; t <= dim_T; ++t) {
            if (r == round && t > level) break;
            if (active(r, t)) ++step;
        }
    const int z = round - 2 * R * level;
    if (z_out) *z_out = z;
    if (slot_out) *slot_out = z % (2 * R + 2);
    return step;
}
