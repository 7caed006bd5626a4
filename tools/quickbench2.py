"""7pt throughput for chosen (n, D, variant) triples: python tools/quickbench2.py n:D:variant ..."""
import sys, time
sys.path.insert(0, '.')
import torch, paper_conf_sc_nguyensckd10_b200 as st
for c in sys.argv[1:]:
    n, D, v = (int(t) for t in c.split(':'))
    try:
        p = st.Plan(n, n, n, torch.float32, D)
        p.set_option(st.ST_OPT_ST7_VARIANT, v)
        i = p.info()
    except Exception as e:
        print(c, 'ERR', e); continue
    x = torch.rand(n, n, n, device='cuda'); y = torch.empty_like(x)
    T = 100 - 100 % D if D != 3 else 99
    p.st7(x, y, 0.4, 0.1, T); p.sync()
    ts = []
    for _ in range(3):
        t0 = time.time(); p.st7(x, y, 0.4, 0.1, T); p.sync(); ts.append(time.time() - t0)
    t = min(ts)
    print(f"{c:16s} tile {i['tile_x']}x{i['tile_y']} thr {i['threads']} k={i['kappa']:.3f} ring {i['ring']}  "
          f"{(n-2)**3*T/t/1e9:7.1f} Gupd/s", flush=True)
    p.close()
