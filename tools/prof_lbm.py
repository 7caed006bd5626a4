import sys; sys.path.insert(0, '.')
import torch, stgen, paper_conf_sc_nguyensckd10_b200 as st
n = int(sys.argv[1]); D = int(sys.argv[2]); T = int(sys.argv[3])
fl = torch.from_numpy(stgen.cavity_flags(n, n, n)).cuda()
f = torch.from_numpy(stgen.lbm_rest(n, n, n, 'float32')).cuda(); g = torch.empty_like(f)
p = st.Plan(n, n, n, torch.float32, D); p.lbm(f, g, 1.6, T, fl); p.sync(); print(p.info(True))
