import sys; sys.path.insert(0, '.')
import numpy as np, torch, stgen, paper_conf_sc_nguyensckd10_b200 as st
n = int(sys.argv[1]) if len(sys.argv) > 1 else 64
D = int(sys.argv[2]) if len(sys.argv) > 2 else 2
a = stgen.grid7(n, n, n, 1, np.float32)
p = st.Plan(n, n, n, torch.float32, D)
x = torch.from_numpy(a).cuda(); y = torch.empty_like(x)
p.st7(x, y, 0.4, 0.1, 4); p.sync(); print("ok", p.info())
