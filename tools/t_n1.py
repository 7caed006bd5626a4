import sys; sys.path.insert(0, '.')
import numpy as np, torch, stgen, paper_conf_sc_nguyensckd10_b200 as st
var = int(sys.argv[1]); D = int(sys.argv[2])
nx, ny, nz = 64, 64, 12
a = stgen.grid7(nx, ny, nz, 7, np.float32)
with st.Plan(nx, ny, nz, torch.float32, D) as p:
    p.set_option(st.ST_OPT_ST7_VARIANT, var)
    print(p.info())
    x = torch.from_numpy(a).cuda(); y = torch.empty_like(x)
    p.st7(x, y, 0.4, 0.1, D); p.sync()
print('ok')
