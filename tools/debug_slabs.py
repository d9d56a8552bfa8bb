import math, os, sys
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd
LAM = 1 / math.sqrt(3)
dims = (45, 38, 31)
MB = int(sys.argv[1]) if len(sys.argv) > 1 else 3
mask_t = I.make_mask("dome", *dims)
mm = I.material_map(mask_t, "region", 8).numpy(); mask = mask_t.numpy()
if MB:
    beta0, D, E, F = I.fd_tables(8, MB, seed=2)
else:
    beta0, D, E, F = [0.1]*8, None, None, None
rng = np.random.default_rng(2)
up = rng.uniform(-1, 1, mask.shape).astype(np.float32); uc = rng.uniform(-1, 1, mask.shape).astype(np.float32)
whole = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
plan = rafd.rafd_slab_plan(mask, 32, MB, 2)
print("plan", plan)
slabs = [rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=k, nranks=2, z_begin=a, z_end=b) for k, (a, b) in enumerate(plan)]
for r in [whole] + slabs:
    r.set_state(up, uc)
cs = np.concatenate([s.read_field()[0] for s in slabs]); cw = whole.read_field()[0]
print("after set_state equal:", np.array_equal(cw, cs))
for st in range(4):
    whole.step(1); rafd.rafd_step_group(slabs, 1)
    cw = whole.read_field()[0]; cs = np.concatenate([s.read_field()[0] for s in slabs])
    bad = np.argwhere(cw != cs)
    print("step", st, "mismatches", len(bad), "planes", sorted(set(bad[:, 0].tolist()))[:10], bad[:3].tolist())
Kw = whole.get_classification()[0]
Ks = np.concatenate([s.get_classification()[0] for s in slabs])
print("K equal", np.array_equal(Kw, Ks), np.argwhere(Kw != Ks)[:5].tolist())
# fresh: one step from the initial state; difference pattern at plane z0-1 of slab 1
whole = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
slabs = [rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=k, nranks=2, z_begin=a, z_end=b) for k, (a, b) in enumerate(plan)]
for r in [whole] + slabs:
    r.set_state(np.zeros_like(up), np.zeros_like(uc))
z0 = plan[1][0]
uc2 = np.zeros_like(uc); uc2[z0 - 1, 10, 20] = 1.0   # impulse in slab 0's top plane
for r in [whole] + slabs:
    r.set_state(None, uc2)
whole.step(1); rafd.rafd_step_group(slabs, 1)
cw = whole.read_field()[0]; cs = np.concatenate([s.read_field()[0] for s in slabs])
print("impulse at z0-1: whole nonzeros", np.argwhere(cw != 0).tolist())
print("slabs nonzeros", np.argwhere(cs != 0).tolist())
print(cw[z0, 10, 20], cs[z0, 10, 20], cw[z0-1,10,20], cs[z0-1,10,20])
