"""Run one radius-2 sweep config for ncu capture: python tools/prof_st13.py N dtype D T"""
import sys; sys.path.insert(0, '.')
import torch, paper_conf_sc_nguyensckd10_b200 as st
n = int(sys.argv[1]); dt = torch.float32 if sys.argv[2] == 'f32' else torch.float64
D = int(sys.argv[3]); T = int(sys.argv[4])
p = st.Plan(n, n, n, dt, D)
x = torch.rand(n, n, n, dtype=dt, device='cuda'); y = torch.empty_like(x)
p.st13(x, y, 0.625, 0.05 * 4 / 3, -0.05 / 12, T); p.sync()
print('ok')
