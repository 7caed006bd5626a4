"""Small runs of every kernel family for compute-sanitizer (racecheck / synccheck /
memcheck / initcheck): python tools/sanitize_driver.py [st7|st13|st27|lbm|all]
Each case runs T = 2 sweeps of depth D at 64^3 (LBM 32x24x20) and checks
the result against the oracle, so a tool-induced change would also show."""
import sys
sys.path.insert(0, '.')
import numpy as np
import torch
import stgen
import oracle
import paper_conf_sc_nguyensckd10_b200 as st

which = sys.argv[1] if len(sys.argv) > 1 else 'all'


def rel(g, o):
    return float(np.max(np.abs(g.astype(np.float64) - o) / np.maximum(np.abs(o.astype(np.float64)), 1e-30)))


fails = 0
if which in ('st7', 'all'):
    for dt, Ds in ((np.float32, range(1, 9)), (np.float64, range(1, 9))):
        a = stgen.grid7(64, 48, 24, 5, dt)
        for D in Ds:
            T = 2 * D + 1
            ref = oracle.st7(a, 0.4, 0.1, T)
            with st.Plan(64, 48, 24, torch.float32 if dt == np.float32 else torch.float64, D) as p:
                x = torch.from_numpy(a).cuda(); y = torch.empty_like(x)
                p.st7(x, y, 0.4, 0.1, T); p.sync()
                e = rel(y.cpu().numpy(), ref)
            ok = e <= (1e-5 if dt == np.float32 else 1e-12)
            fails += not ok
            print(f"st7 {np.dtype(dt).name} D={D} T={T} rel={e:.2e} {'ok' if ok else 'FAIL'}", flush=True)
if which in ('st27', 'all'):
    W = (0.5, 0.04, 0.02, 0.01)
    for dt, Ds in ((np.float32, range(1, 5)), (np.float64, range(1, 3))):
        a = stgen.grid7(64, 40, 20, 6, dt)
        for D in Ds:
            T = 2 * D + 1
            ref = oracle.st27(a, *W, T)
            with st.Plan(64, 40, 20, torch.float32 if dt == np.float32 else torch.float64, D) as p:
                p.set_bitexact(True)
                x = torch.from_numpy(a).cuda(); y = torch.empty_like(x)
                p.st27(x, y, *W, T); p.sync()
                ok = np.array_equal(y.cpu().numpy(), ref)
            fails += not ok
            print(f"st27 {np.dtype(dt).name} D={D} T={T} {'ok' if ok else 'FAIL'}", flush=True)
if which in ('st13', 'all'):
    W13 = (0.625, 0.05 * 4 / 3, -0.05 / 12)
    for dt, Ds in ((np.float32, range(1, 5)), (np.float64, range(1, 4))):
        a = stgen.grid7(64, 40, 24, 8, dt)
        for D in Ds:
            T = 2 * D + 1
            ref = oracle.st13(a, *W13, T)
            with st.Plan(64, 40, 24, torch.float32 if dt == np.float32 else torch.float64, D) as p:
                p.set_bitexact(True)
                x = torch.from_numpy(a).cuda(); y = torch.empty_like(x)
                p.st13(x, y, *W13, T); p.sync()
                ok = np.array_equal(y.cpu().numpy(), ref)
            fails += not ok
            print(f"st13 {np.dtype(dt).name} D={D} T={T} {'ok' if ok else 'FAIL'}", flush=True)
if which in ('lbm', 'all'):
    nx, ny, nz = 32, 24, 20
    flags = stgen.cavity_flags(nx, ny, nz)
    for dt in (np.float32, np.float64):
        f0 = stgen.lbm_random(nx, ny, nz, 3, dt)
        for D, kern in ((1, 1), (2, 2), (3, 2)):
            if dt == np.float64 and D == 3:
                continue
            T = 2 * D + 1
            ref = oracle.lbm(f0, flags, 1.6, T)
            with st.Plan(nx, ny, nz, torch.float32 if dt == np.float32 else torch.float64, D) as p:
                p.set_bitexact(True)
                p.set_option(st.ST_OPT_LBM_KERNEL, kern)
                a = torch.from_numpy(f0).cuda(); b = torch.empty_like(a)
                p.lbm(a, b, 1.6, T, torch.from_numpy(flags).cuda()); p.sync()
                ok = np.array_equal(b.cpu().numpy(), ref)
            fails += not ok
            print(f"lbm {np.dtype(dt).name} D={D} kernel={kern} T={T} {'ok' if ok else 'FAIL'}", flush=True)
print("FAILURES", fails)
sys.exit(1 if fails else 0)
