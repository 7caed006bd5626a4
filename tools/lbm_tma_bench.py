"""LBM kernel A/B on the GPU: push (ST_OPT_LBM_KERNEL 1), gather form (3) and the
TMA-fed gather form (4) at several ring depths; 256^3 cavity, T steps, CUDA events.
python tools/lbm_tma_bench.py [n] [T]"""
import sys
sys.path.insert(0, '.')
import torch
import stgen
import paper_conf_sc_nguyensckd10_b200 as st

n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
T = int(sys.argv[2]) if len(sys.argv) > 2 else 40
only = sys.argv[3] if len(sys.argv) > 3 else ''
for dt, npdt, E in ((torch.float32, 'float32', 4), (torch.float64, 'float64', 8)):
    if only and only != npdt:
        continue
    fl = torch.from_numpy(stgen.cavity_flags(n, n, n)).cuda()
    f = torch.from_numpy(stgen.lbm_rest(n, n, n, npdt)).cuda()
    g = torch.empty_like(f)
    cfgs = [(1, 0), (3, 0)] + [(4, s) for s in ((1, 2, 3, 4, 5) if E == 4 else (1, 2, 3, 4))]
    if n > 512:
        cfgs = [(1, 0), (4, 3), (4, 4)]
    for kern, stages in cfgs:
        p = st.Plan(n, n, n, dt, 1)
        p.set_option(st.ST_OPT_LBM_KERNEL, kern)
        if stages:
            p.set_option(st.ST_OPT_LBM_STAGES, stages)
        p.set_stream(torch.cuda.current_stream())
        try:
            p.lbm(f, g, 1.6, 4, fl)
        except Exception as e:
            print(f"{npdt} kernel {kern} stages {stages}: {e}")
            p.close()
            continue
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        p.lbm(f, g, 1.6, T, fl)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        glups = (n - 2) ** 3 * T / (ms * 1e-3) / 1e9
        gbs = n ** 3 * (38 * E + 1) * T / (ms * 1e-3) / 1e9
        print(f"{npdt} kernel {kern} stages {stages}: {glups:.2f} GLUPS, {gbs:.0f} GB/s "
              f"({ms / T * 1e3:.1f} us/step)", flush=True)
        p.close()
