"""quick 7pt throughput table: python tools/quickbench.py [variant ...]
variant = VY*1000 + threads (st_plan_set_option ST_OPT_ST7_VARIANT), 0 = planner default"""
import sys, time
sys.path.insert(0, '.')
import torch, paper_conf_sc_nguyensckd10_b200 as st
variants = [int(v) for v in sys.argv[1:]] or [0]
cases = [(256, torch.float32, d) for d in (1, 2, 3, 4, 5, 6)] + [(512, torch.float32, d) for d in (3, 4, 5, 6)] + \
        [(256, torch.float64, d) for d in (2, 3, 4)]
for v in variants:
    for (n, dt, D) in cases:
        try:
            p = st.Plan(n, n, n, dt, D)
            p.set_option(st.ST_OPT_ST7_VARIANT, v)
            i = p.info()
        except Exception as e:
            print(v, n, dt, D, 'ERR', e); continue
        x = torch.rand(n, n, n, dtype=dt, device='cuda'); y = torch.empty_like(x)
        T = 100 - 100 % D if D != 3 else 99
        p.st7(x, y, 0.4, 0.1, T); p.sync()
        ts = []
        for _ in range(3):
            t0 = time.time(); p.st7(x, y, 0.4, 0.1, T); p.sync(); ts.append(time.time() - t0)
        t = min(ts)
        print(f"{v:5d} {n} {str(dt)[6:]} D={D} tile {i['tile_x']}x{i['tile_y']} thr {i['threads']} k={i['kappa']:.3f} "
              f"var {i['kernel']} ring {i['ring']}  {t*1e3:7.2f} ms {(n-2)**3*T/t/1e9:7.1f} Gupd/s", flush=True)
        p.close()
