"""27-point GPU vs oracle mismatch map (debug helper)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import stgen, oracle
import paper_conf_sc_nguyensckd10_b200 as st
W = (0.3, 0.05, 0.02, 0.01)
for (n, T, D, ex) in [(64, 1, 1, True), (64, 1, 1, False), (64, 2, 2, True), (64, 4, 2, False), (40, 1, 1, True), (32, 1, 1, True)]:
    a = stgen.grid7(n, n, n, 1, np.float32)
    ref = oracle.st27(a, *W, T)
    with st.Plan(n, n, n, torch.float32, D) as p:
        p.set_bitexact(ex)
        x = torch.from_numpy(a).cuda(); y = torch.zeros_like(x)
        p.st27(x, y, *W, T); p.sync()
        g = y.cpu().numpy()
    bad = np.argwhere(np.abs(g.astype(np.float64) - ref) > 1e-5 * np.abs(ref) + 1e-30)
    print(n, T, D, ex, "bad", len(bad), "of", g.size)
    if len(bad):
        for ax, name in ((0, "z"), (1, "y"), (2, "x")):
            print("  ", name, np.unique(bad[:, ax])[:40])
        z, y_, x_ = bad[0]
        print("  first", bad[0], g[z, y_, x_], ref[z, y_, x_], "input", a[z, y_, x_])
