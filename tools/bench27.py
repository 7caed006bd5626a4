"""Quick 27-point timing: Gupd/s at 256^3 (or argv[1]) for every depth, FP32 and FP64."""
import sys
import numpy as np
import torch
sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
import stgen
import paper_conf_sc_nguyensckd10_b200 as st

n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
T = 100
for dt_np, tdt, dmax in ((np.float32, torch.float32, 4), (np.float64, torch.float64, 4)):
    x = torch.from_numpy(stgen.grid7(n, n, n, 2, dt_np)).cuda()
    y = torch.empty_like(x)
    for d in range(1, dmax + 1):
        with st.Plan(n, n, n, tdt, d) as p:
            p.st27(x, y, 0.3, 0.05, 0.02, 0.01, T)
            p.sync()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s = torch.cuda.current_stream()
            ms = []
            for _ in range(3):
                torch.cuda.synchronize()
                e0.record(); p.st27(x, y, 0.3, 0.05, 0.02, 0.01, T); p.sync(); e1.record(); e1.synchronize()
                ms.append(e0.elapsed_time(e1))
            print(dt_np.__name__, "D", d, "ms", round(min(ms), 3), "Gupd/s", round((n - 2) ** 3 * T / min(ms) / 1e6, 1), flush=True)
