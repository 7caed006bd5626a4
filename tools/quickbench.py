import time, torch, numpy as np, sys
sys.path.insert(0,'.')
import paper_conf_sc_nguyensckd10_b200 as st, stgen
for (n, dt, D) in [(256, torch.float32, 1),(256, torch.float32, 2),(256, torch.float32, 4),(512, torch.float32, 4),(512, torch.float32, 3),(512, torch.float32, 5),(512, torch.float32, 6),(256, torch.float64, 2)]:
    p = st.Plan(n,n,n,dt,D)
    x = torch.rand(n,n,n,dtype=dt,device='cuda'); y=torch.empty_like(x)
    T = 100 if D != 3 else 99
    p.st7(x,y,0.4,0.1,T); p.sync()
    s=torch.cuda.Event(enable_timing=True); e=torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); s.record(torch.cuda.current_stream())
    t0=time.time(); p.st7(x,y,0.4,0.1,T); p.sync(); t1=time.time()
    upd = (n-2)**3*T
    print(n, dt, D, p.info(), f"{(t1-t0)*1e3:.2f} ms  {upd/(t1-t0)/1e9:.1f} Gupd/s", flush=True)
    p.close()
