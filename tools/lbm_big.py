"""LBM FP32 cavity throughput on big lattices (device-built): python tools/lbm_big.py NX NY NZ [T]"""
import sys, time; sys.path.insert(0, '.')
import numpy as np, torch, stgen, paper_conf_sc_nguyensckd10_b200 as st
nx, ny, nz = (int(a) for a in sys.argv[1:4]); T = int(sys.argv[4]) if len(sys.argv) > 4 else 10
fl = torch.zeros((nz, ny, nx), dtype=torch.uint8, device="cuda")
fl[:, 0, :] = 1; fl[:, :, 0] = 1; fl[:, :, nx - 1] = 1; fl[0] = 1; fl[nz - 1] = 1; fl[:, ny - 1, :] = 2
f = torch.empty((19, nz, ny, nx), dtype=torch.float32, device="cuda")
w = stgen.lbm_rest(1, 1, 1, np.float32).reshape(19)
for i in range(19): f[i].fill_(float(w[i]))
g = torch.empty_like(f)
with st.Plan(nx, ny, nz, torch.float32, 1) as p:
    p.lbm(f, g, 1.6, 2, fl); p.sync()
    dt = 1e9
    for _ in range(2):
        t0 = time.time(); p.lbm(f, g, 1.6, T, fl); p.sync(); dt = min(dt, time.time() - t0)
print(f"lbm f32 {nx}x{ny}x{nz}: {(nx-2)*(ny-2)*(nz-2)*T/dt/1e9:.2f} GLUPS  pop stride {nx*ny*nz*4/2**20:.0f} MiB")
