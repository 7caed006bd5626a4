import sys; sys.path.insert(0, '.')
import numpy as np, torch, stgen, oracle, paper_conf_sc_nguyensckd10_b200 as st
ok = True
for var in (214512, 214256):
    for (nx, ny, nz) in ((68, 52, 37), (200, 70, 11), (64, 130, 9), (16, 9, 5), (128, 96, 20)):
        for D in (1, 2, 3, 4):
            a = stgen.grid7(nx, ny, nz, 7, np.float32); T = 2 * D + 1
            ref = oracle.st7(a, 0.4, 0.1, T)
            for ex in (True, False):
                with st.Plan(nx, ny, nz, torch.float32, D) as p:
                    p.set_bitexact(ex); p.set_option(st.ST_OPT_ST7_VARIANT, var)
                    x = torch.from_numpy(a).cuda(); y = torch.empty_like(x)
                    p.st7(x, y, 0.4, 0.1, T); p.sync(); g = y.cpu().numpy()
                good = np.array_equal(g, ref) if ex else np.max(np.abs(g - ref) / np.maximum(np.abs(ref), 1e-30)) <= 1e-5
                if not good: ok = False; print('FAIL', var, nx, ny, nz, D, ex)
print('narrow parity', 'OK' if ok else 'FAILED')
