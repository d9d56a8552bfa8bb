import math, sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import bench
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd
LAM = 1 / math.sqrt(3)
cfg = bench.workload("C4", 1)
nx, ny, nz = cfg["room"]
beta0, D, E, F = I.config_materials(cfg)
dev = torch.device("cuda", 0)
mask_d, mm_d, _ = bench.slab_inputs(cfg, 0, nz, dev)
rooms = {}
for name, tb, dyn in (("tb1", 1, None), ("tb2dyn", 2, "1"), ("tb2stat", 2, "0")):
    pass
g = rafd.Room(mask_d, LAM, 32, beta0, D, E, F, matmap=mm_d)
g2 = rafd.Room(mask_d, LAM, 32, beta0, D, E, F, matmap=mm_d)
g2.set_temporal_blocking(2)
nb = g.nb
gen = torch.Generator(device=dev).manual_seed(20251017)
up = torch.rand((nz, ny, nx), generator=gen, device=dev, dtype=torch.float32) * 2 - 1
uc = torch.rand((nz, ny, nx), generator=gen, device=dev, dtype=torch.float32) * 2 - 1
v0 = (torch.rand((3, nb), generator=gen, device=dev, dtype=torch.float32) - 0.5) * 0.2
g0 = (torch.rand((3, nb), generator=gen, device=dev, dtype=torch.float32) - 0.5) * 0.2
src = I.source_position((nx, ny, nz))
for r in (g, g2):
    r.set_state(up, uc, v0, g0)
    r.set_source(src, [1.0, -0.5])
    r.step(2)
    r.synchronize()
f = []
for r in (g, g2):
    c = torch.empty((nz, ny, nx), dtype=torch.float32, device=dev)
    p = torch.empty_like(c)
    r.read_field(out_curr=c, out_prev=p)
    f.append((c, p))
d = (f[0][0] != f[1][0])
print("cur differ:", int(d.sum()), "prev differ:", int((f[0][1] != f[1][1]).sum()))
if d.any():
    idx = d.nonzero()[:10]
    print(idx.tolist())
    zs = d.nonzero()[:, 0]
    print("z range", int(zs.min()), int(zs.max()))
    ys = d.nonzero()[:, 1]; xs = d.nonzero()[:, 2]
    print("y range", int(ys.min()), int(ys.max()), "x range", int(xs.min()), int(xs.max()))
# compare tb1 with a fresh tb1 to make sure g is deterministic
print("info", g2.get_info()["steps"], g.get_info()["steps"])
