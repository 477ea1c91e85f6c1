import time, sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_icde_doraiswamyf22_b200 as sp
from gen import configs
sp.load()
w = configs.pp()
dA = {k: torch.as_tensor(np.ascontiguousarray(v)).cuda() for k, v in w.polys.items()}
dB = {k: torch.as_tensor(np.ascontiguousarray(v)).cuda() for k, v in w.polys2.items()}
ts = []
for i in range(30):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    sp.join_polygons(dA, dB, max_dim=w.max_dim)
    torch.cuda.synchronize(); ts.append(1e3 * (time.perf_counter() - t0))
print("pp per-call ms:", [round(t, 1) for t in ts])
cv = sp.Canvas(w.polys, max_dim=8192)
ts = []
for i in range(10):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    c = sp.Canvas(w.polys, max_dim=8192); c.close()
    torch.cuda.synchronize(); ts.append(1e3 * (time.perf_counter() - t0))
print("build+free ms:", [round(t, 1) for t in ts])
