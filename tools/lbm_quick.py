"""quick LBM throughput: python tools/lbm_quick.py [n] [D ...]; env ST_LBM_PUSH1=1 selects the per-neighbour-flag push kernel"""
import sys, time; sys.path.insert(0, '.')
import torch, stgen, paper_conf_sc_nguyensckd10_b200 as st
n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
Ds = [int(a) for a in sys.argv[2:]] or [1, 2, 3]
for dt, npdt in ((torch.float32, 'float32'), (torch.float64, 'float64')):
    fl = torch.from_numpy(stgen.cavity_flags(n, n, n)).cuda()
    f = torch.from_numpy(stgen.lbm_rest(n, n, n, npdt)).cuda(); g = torch.empty_like(f)
    for D in Ds:
        try:
            p = st.Plan(n, n, n, dt, D)
        except Exception as e:
            print(D, e); continue
        T = 40
        p.lbm(f, g, 1.6, T, fl); p.sync()
        t0 = time.time(); p.lbm(f, g, 1.6, T, fl); p.sync(); t1 = time.time()
        print(f"lbm {npdt} D={D} {(n-2)**3*T/(t1-t0)/1e9:.2f} GLUPS  ({(t1-t0)/T*1e3:.3f} ms/step)", flush=True)
        p.close()
