"""LBM throughput through the Z-slab schedule on one GPU (loopback slabs): TMA gather vs push.
python tools/lbm_slab_speed.py"""
import sys; sys.path.insert(0,'.')
import torch, stgen, paper_conf_sc_nguyensckd10_b200 as st
n=256; T=40
fl=torch.from_numpy(stgen.cavity_flags(n,n,n)).cuda()
f=torch.from_numpy(stgen.lbm_rest(n,n,n,'float32')).cuda(); g=torch.empty_like(f)
for slabs, kern in ((1,0),(2,0),(4,0),(2,1),(4,1)):
    p=st.Plan(n,n,n,torch.float32,1)
    if kern: p.set_option(st.ST_OPT_LBM_KERNEL, kern)
    if slabs>1: st.st_plan_set_loopback_slabs(p.h, slabs)
    p.lbm(f,g,1.6,4,fl); p.sync()
    import time
    p.sync(); torch.cuda.synchronize(); t0=time.perf_counter(); p.lbm(f,g,1.6,T,fl); p.sync(); ms=(time.perf_counter()-t0)*1e3
    print(f"slabs {slabs} kernel {p.info(True)['kernel']}: {(n-2)**3*T/(ms*1e-3)/1e9:.2f} GLUPS"); p.close()
