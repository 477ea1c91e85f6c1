# Cold vs warm canvas build of C5 (first build in a process pays CUDA module loading and pool growth).
import time, os, sys
sys.path.insert(0, os.getcwd())
import torch, numpy as np
import paper_conf_icde_doraiswamyf22_b200 as sp
from gen import configs
t0=time.perf_counter(); w = configs.c5(); t1=time.perf_counter()
print("workload gen (host)", round(t1-t0,3))
torch.cuda.init(); torch.zeros(1, device='cuda'); torch.cuda.synchronize()
sp.load()
t0=time.perf_counter()
a=torch.as_tensor(w.polys['ring_xy']).cuda(); b=torch.as_tensor(w.polys['ring_off']).cuda(); c=torch.as_tensor(w.polys['poly_ring_off']).cuda(); torch.cuda.synchronize()
print("H2D polygons", round(time.perf_counter()-t0,3), a.numel()*4/1e6, "MB")
for i in range(3):
    torch.cuda.synchronize(); t0=time.perf_counter()
    cv=sp.Canvas(w.polys, max_dim=w.max_dim); torch.cuda.synchronize()
    print("build", i, round(time.perf_counter()-t0,3), cv.build_times())
    cv.close()
