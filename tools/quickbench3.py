"""7pt throughput on nx x ny x nz grids: python tools/quickbench3.py nx:ny:nz:D:variant ..."""
import sys, time
sys.path.insert(0, '.')
import torch, paper_conf_sc_nguyensckd10_b200 as st
for c in sys.argv[1:]:
    nx, ny, nz, D, v = (int(t) for t in c.split(':'))
    p = st.Plan(nx, ny, nz, torch.float32, D)
    p.set_option(st.ST_OPT_ST7_VARIANT, v)
    i = p.info()
    x = torch.rand(nz, ny, nx, device='cuda'); y = torch.empty_like(x)
    T = 8 * D if D != 3 else 24
    p.st7(x, y, 0.4, 0.1, T); p.sync()
    ts = []
    for _ in range(3):
        t0 = time.time(); p.st7(x, y, 0.4, 0.1, T); p.sync(); ts.append(time.time() - t0)
    t = min(ts)
    run = i['tiles_x'] * i['tiles_y'] * (nz - 2) / 148
    print(f"{c:22s} tiles {i['tiles_x']}x{i['tiles_y']} k={i['kappa']:.3f} thr {i['threads']} planes/CTA {run:6.1f}  "
          f"{(nx-2)*(ny-2)*(nz-2)*T/t/1e9:7.1f} Gupd/s", flush=True)
    p.close()
