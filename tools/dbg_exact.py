import sys; sys.path.insert(0,'.')
import numpy as np, torch, oracle, stgen, paper_conf_sc_nguyensckd10_b200 as st
a = stgen.grid7(64,64,64,1,np.float32)
for T in (1,2,4):
  ref = oracle.st7(a,0.4,0.1,T)
  for D in (1,2):
    p = st.Plan(64,64,64,torch.float32,D); p.set_bitexact(True)
    x=torch.from_numpy(a).cuda(); y=torch.empty_like(x); p.st7(x,y,0.4,0.1,T); p.sync(); g=y.cpu().numpy()
    d = np.argwhere(g!=ref)
    print("T",T,"D",D,"ndiff",len(d), d[:5].tolist(), [(float(g[tuple(i)]),float(ref[tuple(i)])) for i in d[:3]])
    p.close()
# manual: one interior point, T=1
al=np.float32(0.4); be=np.float32(0.1)
z,y,x=5,5,5
c=a[z,y,x]; s=((a[z,y,x-1]+a[z,y,x+1])+(a[z,y-1,x]+a[z,y+1,x]))+(a[z-1,y,x]+a[z+1,y,x])
print("manual", al*c+be*s, oracle.st7(a,0.4,0.1,1)[z,y,x], np.float32(np.fma(al,c,be*s)) if hasattr(np,'fma') else None)
