import sys, time; sys.path.insert(0, '.')
import torch, stgen, paper_conf_sc_nguyensckd10_b200 as st
n = 256
for dt, npdt in ((torch.float32, 'float32'), (torch.float64, 'float64')):
    fl = torch.from_numpy(stgen.cavity_flags(n, n, n)).cuda()
    f = torch.from_numpy(stgen.lbm_rest(n, n, n, npdt)).cuda(); g = torch.empty_like(f)
    for D in (1, 2, 3):
        try:
            p = st.Plan(n, n, n, dt, D)
        except Exception as e:
            print(D, e); continue
        T = 12
        p.lbm(f, g, 1.6, T, fl); p.sync()
        t0 = time.time(); p.lbm(f, g, 1.6, T, fl); p.sync(); t1 = time.time()
        print(f"lbm {npdt} D={D} info={p.info(True)} {(n-2)**3*T/(t1-t0)/1e9:.2f} GLUPS", flush=True)
        p.close()
