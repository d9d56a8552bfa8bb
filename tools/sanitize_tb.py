"""Temporal blocking under compute-sanitizer: a whole room with two steps per
sweep and the same room as 3 z slabs (rafd_step_group, temporal blocking in
every slab), 7 steps each (3 double steps + 1 single), compared bitwise.
    compute-sanitizer --tool memcheck python tools/sanitize_tb.py [prec] [MB] [n] [shape]"""
import math
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd  # noqa: E402

prec = int(sys.argv[1]) if len(sys.argv) > 1 else 32
MB = int(sys.argv[2]) if len(sys.argv) > 2 else 3
n = int(sys.argv[3]) if len(sys.argv) > 3 else 16
shape = sys.argv[4] if len(sys.argv) > 4 else "dome"
dims = (3 * n + 7, 2 * n + 3, n)
mask = I.make_mask(shape, *dims).numpy()
if MB:
    b0, D, E, F = I.fd_tables(2, MB)
else:
    b0, D, E, F = [0.1, 0.2], None, None, None
mm = I.material_map(I.torch.from_numpy(mask), "random", 2).numpy()
lam = 1 / math.sqrt(3)
src = I.snap_inside(mask, (n // 2, n // 2, n // 2))
whole = rafd.Room(mask, lam, prec, b0, D, E, F, matmap=mm)
whole.set_temporal_blocking(2)
plan = rafd.rafd_slab_plan(mask, prec, MB, 3)
slabs = [rafd.Room(mask, lam, prec, b0, D, E, F, matmap=mm, rank=k, nranks=3, z_begin=a, z_end=b)
         for k, (a, b) in enumerate(plan)]
for r in [whole] + slabs:
    if r is not whole:
        r.set_temporal_blocking(2)
    r.set_source(src, I.gaussian_pulse(8, 2.0))
whole.step(7)
rafd.rafd_step_group(slabs, 7)
cw = whole.read_field()[0]
cs = np.concatenate([s.read_field()[0] for s in slabs])
assert np.array_equal(cw, cs), "slabs differ from the whole room"
print("ok", plan, np.abs(cw).sum())
