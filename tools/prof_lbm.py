"""one LBM run for ncu: python tools/prof_lbm.py N D T [f32|f64]"""
import sys; sys.path.insert(0, '.')
import torch, stgen, paper_conf_sc_nguyensckd10_b200 as st
n = int(sys.argv[1]); D = int(sys.argv[2]); T = int(sys.argv[3])
dt = sys.argv[4] if len(sys.argv) > 4 else 'f32'
tt, nd = (torch.float32, 'float32') if dt == 'f32' else (torch.float64, 'float64')
fl = torch.from_numpy(stgen.cavity_flags(n, n, n)).cuda()
f = torch.from_numpy(stgen.lbm_rest(n, n, n, nd)).cuda(); g = torch.empty_like(f)
p = st.Plan(n, n, n, tt, D); p.lbm(f, g, 1.6, T, fl); p.sync(); print(p.info(True))
