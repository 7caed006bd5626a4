"""quick 7pt throughput table: python tools/quickbench.py [variant ...]  (ST_VARIANT env is read per plan)"""
import os, sys, time
sys.path.insert(0, '.')
import torch, paper_conf_sc_nguyensckd10_b200 as st
variants = sys.argv[1:] or ['']
cases = [(256, torch.float32, d) for d in (2, 3, 4, 5, 6)] + [(512, torch.float32, d) for d in (3, 4, 5)] + \
        [(256, torch.float64, d) for d in (2, 3, 4)]
for v in variants:
    if v: os.environ['ST_VARIANT'] = v
    else: os.environ.pop('ST_VARIANT', None)
    for (n, dt, D) in cases:
        try:
            p = st.Plan(n, n, n, dt, D)
        except Exception as e:
            print(v, n, dt, D, 'ERR', e); continue
        x = torch.rand(n, n, n, dtype=dt, device='cuda'); y = torch.empty_like(x)
        T = 100 - 100 % D if D != 3 else 99
        p.st7(x, y, 0.4, 0.1, T); p.sync()
        t0 = time.time(); p.st7(x, y, 0.4, 0.1, T); p.sync(); t1 = time.time()
        i = p.info()
        print(f"{v or 'default':8s} {n} {str(dt)[6:]} D={D} tile {i['tile_x']}x{i['tile_y']} thr {i['threads']} k={i['kappa']:.3f} var {i['kernel']} ring {i['ring']}  {(t1-t0)*1e3:7.2f} ms {(n-2)**3*T/(t1-t0)/1e9:7.1f} Gupd/s", flush=True)
        p.close()
