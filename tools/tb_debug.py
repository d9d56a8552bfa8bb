"""Tiny temporal-blocking run for compute-sanitizer (debug aid)."""
import math
import sys

import numpy as np

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd  # noqa: E402

prec = int(sys.argv[1]) if len(sys.argv) > 1 else 32
n = int(sys.argv[2]) if len(sys.argv) > 2 else 2
mask = I.box_mask(64, 40, 8).numpy()
g = rafd.Room(mask, 1 / math.sqrt(3), prec, np.array([0.2]))
g.set_temporal_blocking(2)
print("info", g.get_info()["n_shell"], flush=True)
g.set_source((10, 10, 4), [1.0])
g.step(n)
g.synchronize()
print("ok", float(np.abs(g.read_field()[0]).sum()))
