"""one LBM run with a chosen kernel for ncu: python tools/prof_lbm_k.py N T f32|f64 KERNEL [STAGES]"""
import sys; sys.path.insert(0, '.')
import torch, stgen, paper_conf_sc_nguyensckd10_b200 as st
n = int(sys.argv[1]); T = int(sys.argv[2]); dt = sys.argv[3]; kern = int(sys.argv[4])
stages = int(sys.argv[5]) if len(sys.argv) > 5 else 0
tt, nd = (torch.float32, 'float32') if dt == 'f32' else (torch.float64, 'float64')
fl = torch.from_numpy(stgen.cavity_flags(n, n, n)).cuda()
f = torch.from_numpy(stgen.lbm_rest(n, n, n, nd)).cuda(); g = torch.empty_like(f)
p = st.Plan(n, n, n, tt, 1); p.set_option(st.ST_OPT_LBM_KERNEL, kern)
if stages: p.set_option(st.ST_OPT_LBM_STAGES, stages)
p.lbm(f, g, 1.6, T, fl); p.sync()
