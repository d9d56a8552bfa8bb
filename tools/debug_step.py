"""Tiny step for debugging kernels under compute-sanitizer: python tools/debug_step.py [prec] [MB] [n]"""
import math
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd  # noqa: E402

prec = int(sys.argv[1]) if len(sys.argv) > 1 else 32
MB = int(sys.argv[2]) if len(sys.argv) > 2 else 0
n = int(sys.argv[3]) if len(sys.argv) > 3 else 20
shape = sys.argv[4] if len(sys.argv) > 4 else "dome"
mask = I.make_mask(shape, 3 * n + 7, 2 * n + 3, n).numpy()
if MB:
    b0, D, E, F = I.fd_tables(2, MB)
else:
    b0, D, E, F = [0.1, 0.2], None, None, None
mm = I.material_map(I.torch.from_numpy(mask), "random", 2).numpy()
r = rafd.Room(mask, 1 / math.sqrt(3), prec, b0, D, E, F, matmap=mm)
r.set_source(I.snap_inside(mask, (n // 2, n // 2, n // 2)), [1.0])
r.step(3)
r.synchronize()
print("ok", np.abs(r.read_field()[0]).sum())
