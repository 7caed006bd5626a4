"""Per-CTA timeline of one 7-point sweep launch (A/B diagnostics build):
  ST_AB=trace ST_AB_DEFS=-DST7_TRACE python -m paper_conf_sc_nguyensckd10_b200.build
  ST35D_LIB=build/ab/trace/libst35d.so python tools/trace7.py n:D[:variant] ...
Prints launch span, per-CTA busy time distribution and per-segment durations."""
import ctypes, sys
sys.path.insert(0, '.')
import numpy as np, torch
import paper_conf_sc_nguyensckd10_b200 as st
L = st.lib()
rd = L.st7_trace_read_f32
for c in sys.argv[1:]:
    f = [int(t) for t in c.split(':')]
    n, D = f[0], f[1]
    nz = f[3] if len(f) > 3 else n
    p = st.Plan(n, n, nz, torch.float32, D)
    if len(f) > 2:
        p.set_option(st.ST_OPT_ST7_VARIANT, f[2])
    x = torch.rand(nz, n, n, device='cuda'); y = torch.empty_like(x)
    for _ in range(3):
        p.st7(x, y, 0.4, 0.1, D); p.sync()
    buf = np.zeros((320, 16), np.uint64)
    assert rd(buf.ctypes.data_as(ctypes.c_void_p)) == 0
    G = 148
    b = buf[:G].astype(np.int64)
    t0 = b[:, 0].min()
    go, end, ns = b[:, 1] - t0, b[:, 12] - t0, b[:, 13]
    span = end.max()
    busy = end - go
    print(f"{c}: span {span/1e3:.1f} us  setup (entry->pdl done) max {go.max()/1e3:.2f} us  "
          f"busy min/med/max {busy.min()/1e3:.1f}/{np.median(busy)/1e3:.1f}/{busy.max()/1e3:.1f} us  "
          f"segments/CTA {np.bincount(ns)}")
    pro, stdy, epi, Ls = [], [], [], []
    for i in range(G):
        k = int(min(ns[i], 3))
        for j in range(k):
            s0, s1, s2 = b[i, 2 + 3 * j], b[i, 3 + 3 * j], b[i, 4 + 3 * j]
            e = b[i, 2 + 3 * (j + 1)] if j + 1 < int(ns[i]) and j + 1 < 3 else (b[i, 12] if j + 1 == int(ns[i]) else 0)
            Lj = (int(b[i, 14]) >> (16 * j)) & 0xffff
            if s1 == 0 or s2 == 0 or e == 0:
                continue
            pro.append(s1 - s0); stdy.append((s2 - s1) / max(Lj, 1)); epi.append(e - s2); Ls.append(Lj)
    pro, stdy, epi, Ls = (np.array(v, float) for v in (pro, stdy, epi, Ls))
    info = p.info()
    Ltot = np.array([sum((int(b[i, 14]) >> (16 * j)) & 0xffff for j in range(min(int(ns[i]), 3))) for i in range(G)])
    order = np.argsort(-busy)
    print("   slowest CTAs (busy us, segments, planes, go us):",
          [(round(busy[i] / 1e3, 1), int(ns[i]), int(Ltot[i]), round(go[i] / 1e3, 2)) for i in order[:8]])
    tile0 = b[:, 15] & 0xffff
    smid = (b[:, 15] >> 16) & 0xffff
    print("   slowest (tile, smid):", [(int(tile0[i]), int(smid[i])) for i in order[:12]])
    print("   fastest (tile, smid):", [(int(tile0[i]), int(smid[i])) for i in order[-12:]])
    tb = {}
    for i in range(G):
        if ns[i] == 1:
            tb.setdefault(int(tile0[i]), []).append(busy[i] / 1e3)
    print("   1-seg busy by tile:", {t: round(float(np.median(v)), 1) for t, v in sorted(tb.items())})
    half = smid < 74
    print(f"   busy med smid<74 {np.median(busy[half & (ns == 1)])/1e3:.1f}  smid>=74 {np.median(busy[~half & (ns == 1)])/1e3:.1f}")
    print("   fastest CTAs:", [(round(busy[i] / 1e3, 1), int(ns[i]), int(Ltot[i])) for i in order[-6:]])
    for k in (1, 2):
        m = ns == k
        if m.any():
            print(f"   {k}-segment CTAs: {m.sum()}  busy med {np.median(busy[m])/1e3:.1f} us  planes med {np.median(Ltot[m]):.0f}"
                  f"  us/plane-equiv {np.median(busy[m] / Ltot[m])/1e3:.3f}")
    print(f"   tiles {info['tiles_x']}x{info['tiles_y']} thr {info['threads']}  segments timed {len(Ls)}  L med {np.median(Ls):.0f}"
          f"  prolog us med {np.median(pro)/1e3:.2f} (max {pro.max()/1e3:.2f})  steady us/plane med {np.median(stdy)/1e3:.3f}"
          f"  epilog us med {np.median(epi)/1e3:.2f}")
    rb = np.zeros((320, 16, 2), np.uint64)
    assert L.st7_trace_rounds_f32(rb.ctypes.data_as(ctypes.c_void_p)) == 0
    rb = rb[:G].astype(np.int64)
    s0 = b[:, 2][:, None]
    land = np.nanmedian(np.where(rb[:, :, 0] > 0, rb[:, :, 0] - s0, np.nan), axis=0) / 1e3
    rend = np.nanmedian(np.where(rb[:, :, 1] > 0, rb[:, :, 1] - s0, np.nan), axis=0) / 1e3
    print("   seg0 rounds (us from segment start, median over CTAs): landed", np.round(land, 2))
    print("                                                         end   ", np.round(rend, 2))
    ib = np.zeros((320, 16), np.uint64)
    assert L.st7_trace_issue_f32(ib.ctypes.data_as(ctypes.c_void_p)) == 0
    ib = ib[:G].astype(np.int64)
    iss = np.nanmedian(np.where(ib > 0, ib - s0, np.nan), axis=0) / 1e3
    print("                                                         issued", np.round(iss, 2))
    p.close()
