"""Short run of the bench workload for ncu (no timing is taken from this).

    ncu ... python tools/profile_run.py [--config C4] [--steps 6]
"""
import argparse
import math
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C4")
ap.add_argument("--dims", default=None, help="nx,ny,nz: a box with the config's materials instead of its room")
ap.add_argument("--steps", type=int, default=6)
ap.add_argument("--graph", action="store_true")
ap.add_argument("--precision", type=int, default=None, choices=[32, 64])
ap.add_argument("--warmup", type=int, default=0, help="untimed steps first (first launches touch fresh pages)")
ap.add_argument("--tb", type=int, default=2, choices=[1, 2], help="steps per sweep (temporal blocking)")
a = ap.parse_args()
cfg = bench.workload(a.config, 1)
if a.dims:
    cfg["room"] = tuple(int(v) for v in a.dims.split(","))
nx, ny, nz = cfg["room"]
if a.precision:
    cfg["precision"] = a.precision
beta0, D, E, F = I.config_materials(cfg)
mask, mm, mz0 = bench.slab_inputs(cfg, 0, nz, torch.device("cuda", 0))
room = rafd.Room(mask, 1 / math.sqrt(3), cfg["precision"], beta0, D, E, F, matmap=mm)
del mask, mm
torch.cuda.empty_cache()
if a.tb == 2:
    room.set_temporal_blocking(2)
room.set_source(I.source_position((nx, ny, nz)), I.impulse())
room.set_receivers(I.receiver_positions((nx, ny, nz)))
if a.warmup:
    room.step(a.warmup)
    room.synchronize()
room.set_profiling(not a.graph)
room.step(a.steps)
room.synchronize()
print("launches", room.launch_count(), room.get_kernel_times())
