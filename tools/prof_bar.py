"""One ablation-ladder bar for an ncu capture: python tools/prof_bar.py NAME [n] [T]
NAME: naive | spatial | 4d | onerow | level | twophase  (FP32 256^3, dim_T 3 unless spatial/naive; T = 9: three sweeps, the 4th launch is a timed dim_T 3 sweep)"""
import sys
sys.path.insert(0, '.')
import torch
import paper_conf_sc_nguyensckd10_b200 as st
name = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 256
T = int(sys.argv[3]) if len(sys.argv) > 3 else 9   # 3 sweeps of dim_T 3
cfg = {"naive": (1, 0, 0, True), "spatial": (1, 0, 0, False), "4d": (3, 0, 64, False),
       "onerow": (3, 1256, 0, False), "level": (3, 94256, 0, False), "twophase": (3, 0, 0, False)}[name]
D, var, zc, naive = cfg
p = st.Plan(n, n, n, torch.float32, D)
if naive:
    p.set_variant(st.ST_VARIANT_NAIVE)
p.set_option(st.ST_OPT_ST7_VARIANT, var)
p.set_option(st.ST_OPT_ZCHUNK, zc)
x = torch.rand(n, n, n, device='cuda'); y = torch.empty_like(x)
p.st7(x, y, 0.4, 0.1, T); p.sync()
print(name, p.info())
