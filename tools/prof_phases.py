"""Per-round phase clocks of the 7-point kernel (ST7_PROF build):
ST35D_LIB=build/ab/prof/libst35d.so python tools/prof_phases.py N D [f32|f64]"""
import os, sys, struct, numpy as np
sys.path.insert(0, '.')
n = int(sys.argv[1]); D = int(sys.argv[2]); dt = sys.argv[3] if len(sys.argv) > 3 else 'f32'
out = f"gpurun_out/prof_{n}_{D}_{dt}.bin"
if os.path.exists(out): os.remove(out)
os.environ["ST_PROF_OUT"] = out
import torch, paper_conf_sc_nguyensckd10_b200 as st
t = torch.float32 if dt == 'f32' else torch.float64
p = st.Plan(n, n, n, t, D)
x = torch.rand(n, n, n, dtype=t, device='cuda'); y = torch.empty_like(x)
p.st7(x, y, 0.4, 0.1, D); p.sync()      # warm
os.remove(out)
p.st7(x, y, 0.4, 0.1, D); p.sync()      # one sweep, profiled
b = open(out, 'rb').read()
grid, wpc, d, nzo = struct.unpack('4i', b[:16])
a = np.frombuffer(b[16:], dtype=np.uint64)[:grid * wpc * 10].reshape(grid, wpc, 10).astype(np.float64)
a = a[:, :max(1, wpc - (1 if a[0, -1, 4] == 0 else 0))]
tot, wait, comp, bar, nr, ns, seg, first, issue, gap = (a[..., i] for i in range(10))
act = nr[..., ] > 0
print(f"N={n} D={d} {dt} grid={grid} warps/cta={wpc}")
print(f"  kernel clocks per CTA: mean {tot[:,0].mean():.0f} max {tot[:,0].max():.0f} min {tot[:,0].min():.0f}")
print(f"  rounds per CTA: mean {nr[:,0].mean():.1f} max {nr[:,0].max():.0f} (steady {ns[:,0].mean():.1f})")
r = nr[:, :].clip(1)
print(f"  per round (mean over warps): wait {(wait/r).mean():.0f}  compute {(comp/r).mean():.0f}  barrier {(bar/r).mean():.0f}  total {(tot/r).mean():.0f}")
print(f"  compute per round by warp (CTA 0): {np.round(comp[0]/r[0]).astype(int).tolist()}")
print(f"  barrier per round by warp (CTA 0): {np.round(bar[0]/r[0]).astype(int).tolist()}")
print(f"  per round: TMA-issue block {(issue/r).mean():.0f} (warp 0: {(issue[:,0]/r[:,0]).mean():.0f}), barrier-end -> next round {(gap/r).mean():.0f}")
print(f"  outside rounds (setup, segment switch) per CTA: {(tot - wait - comp - bar)[:,0].mean():.0f}")
print(f"  segment setup per CTA: {seg[:,0].mean():.0f} (first round starts at {first[:,0].mean():.0f})")
print(f"  rounds per CTA histogram: {np.bincount(nr[:,0].astype(int)).nonzero()[0].tolist()}")
