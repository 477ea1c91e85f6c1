import sys, os
sys.path.insert(0, os.getcwd())
import torch, numpy as np
import gen, paper_conf_icde_doraiswamyf22_b200 as sp
from gen import configs
w = configs.ov(n_points=1_000_000, n_polys=int(sys.argv[1]) if len(sys.argv) > 1 else 1000)
lc = sp.LayeredCanvas(w.polys, max_dim=w.max_dim)
print("layers", lc.num_layers, flush=True)
xy = gen.points_device(w.points, w.point_seed, 0, w.n_points)
c = sp.join_count_layered(lc, xy); torch.cuda.synchronize()
ref = sp.join_count(sp.Canvas(w.polys, max_dim=w.max_dim), xy); torch.cuda.synchronize()
print("equal", bool(torch.equal(c, ref)))
