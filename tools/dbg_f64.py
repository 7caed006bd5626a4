import sys; sys.path.insert(0,'.')
import numpy as np, torch, paper_conf_sc_nguyensckd10_b200 as st
for D in (1,2):
  p = st.Plan(64,64,16,torch.float64,D)
  x=torch.rand(16,64,64,dtype=torch.float64,device='cuda'); y=torch.empty_like(x); p.st7(x,y,0.4,0.1,3); p.sync(); print("ok f64",D,p.info())
