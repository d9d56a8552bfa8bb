"""Wall-clock of room setup with and without temporal blocking (debug aid)."""
import math
import sys
import time

import numpy as np
import torch

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd  # noqa: E402

cfg = bench.workload(sys.argv[1] if len(sys.argv) > 1 else "C3", 1)
prec = int(sys.argv[2]) if len(sys.argv) > 2 else cfg["precision"]
nx, ny, nz = cfg["room"]
beta0, D, E, F = I.config_materials(cfg)
mask, mm, mz0 = bench.slab_inputs(cfg, 0, nz, torch.device("cuda", 0))
for rep in range(2):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    room = rafd.Room(mask, 1 / math.sqrt(3), prec, beta0, D, E, F, matmap=mm)
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    room.set_temporal_blocking(2)
    t2 = time.perf_counter()
    room.set_source(I.source_position((nx, ny, nz)), I.impulse())
    room.set_receivers(I.receiver_positions((nx, ny, nz)))
    t3 = time.perf_counter()
    for _ in range(10):
        room.step(2)
        room.read_receivers(cap=2)
    t4 = time.perf_counter()
    room.destroy()
    t5 = time.perf_counter()
    print(f"rep {rep}: create {t1-t0:.3f} tb {t2-t1:.3f} src/rcv {t3-t2:.3f} 10x(step2+read) {t4-t3:.3f} destroy {t5-t4:.3f}", flush=True)
