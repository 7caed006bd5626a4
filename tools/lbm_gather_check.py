"""gather-form LBM (ST_OPT_LBM_KERNEL 3): parity vs the oracle and throughput vs the push kernel"""
import sys, time
sys.path.insert(0, '.')
import numpy as np, torch, stgen, oracle, paper_conf_sc_nguyensckd10_b200 as st
ok = True
for dt in (np.float32, np.float64):
    for (nx, ny, nz) in ((32, 24, 20), (96, 50, 13)):
        flags = stgen.cavity_flags(nx, ny, nz)
        flags[nz // 2, 5:8, 7:12] = stgen.WALL
        f0 = stgen.lbm_random(nx, ny, nz, 3, dt)
        for T in (1, 2, 5):
            ref = oracle.lbm(f0, flags, 1.6, T)
            for ex in (True, False):
                with st.Plan(nx, ny, nz, torch.float32 if dt == np.float32 else torch.float64, 1) as p:
                    p.set_bitexact(ex); p.set_option(st.ST_OPT_LBM_KERNEL, 3)
                    a = torch.from_numpy(f0).cuda(); b = torch.empty_like(a)
                    p.lbm(a, b, 1.6, T, torch.from_numpy(flags).cuda()); p.sync()
                    g = b.cpu().numpy()
                good = np.array_equal(g, ref) if ex else np.max(np.abs(g - ref) / np.maximum(np.abs(ref), 1e-30)) <= (1e-4 if dt == np.float32 else 1e-12)
                if not good: ok = False; print('FAIL', dt, nx, ny, nz, T, ex)
print('gather parity', 'OK' if ok else 'FAILED', flush=True)
for dt, tdt in ((np.float32, torch.float32), (np.float64, torch.float64)):
    n, T = 256, 20
    fl = torch.from_numpy(stgen.cavity_flags(n, n, n)).cuda()
    f = torch.from_numpy(stgen.lbm_rest(n, n, n, dt)).cuda(); g = torch.empty_like(f)
    for kern in (1, 3):
        with st.Plan(n, n, n, tdt, 1) as p:
            p.set_option(st.ST_OPT_LBM_KERNEL, kern)
            p.lbm(f, g, 1.6, T, fl); p.sync()
            ts = []
            for _ in range(3):
                t0 = time.time(); p.lbm(f, g, 1.6, T, fl); p.sync(); ts.append(time.time() - t0)
            print(np.dtype(dt).name, 'kernel', kern, round((n - 2) ** 3 * T / min(ts) / 1e9, 2), 'GLUPS', flush=True)
