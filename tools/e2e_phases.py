"""Wall-clock breakdown of bench.py's end-to-end leg (create from pinned host
buffers, temporal-blocking enable, source/receivers, the step+read loop,
destroy), to see where the e2e time goes.  python tools/e2e_phases.py [--tb 1|2]"""
import argparse
import math
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--tb", type=int, default=2)
ap.add_argument("--steps", type=int, default=200)
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
cfg = bench.workload("C4", 1)
nx, ny, nz = cfg["room"]
beta0, D, E, F = I.config_materials(cfg)
dev = torch.device("cuda", 0)
mask_d, mm_d, mz0 = bench.slab_inputs(cfg, 0, nz, dev)
mask_h = torch.empty(mask_d.shape, dtype=torch.uint8, pin_memory=True)
mm_h = torch.empty(mm_d.shape, dtype=torch.uint8, pin_memory=True)
mask_h.copy_(mask_d)
mm_h.copy_(mm_d)
del mask_d, mm_d
torch.cuda.empty_cache()
for rep in range(a.reps):
    torch.cuda.synchronize()
    t = [time.perf_counter()]
    room = rafd.Room(mask_h.numpy(), 1 / math.sqrt(3), cfg["precision"], beta0, D, E, F, matmap=mm_h.numpy())
    room.synchronize(); t.append(time.perf_counter())
    if a.tb == 2:
        room.set_temporal_blocking(2)
    room.synchronize(); t.append(time.perf_counter())
    room.set_source(I.source_position((nx, ny, nz)), I.impulse())
    room.set_receivers(I.receiver_positions((nx, ny, nz)))
    room.synchronize(); t.append(time.perf_counter())
    done = 0
    while done < a.steps:
        k = min(a.tb, a.steps - done)
        room.step(k)
        room.read_receivers(cap=k)
        done += k
    room.synchronize(); t.append(time.perf_counter())
    room.destroy(); torch.cuda.synchronize(); t.append(time.perf_counter())
    names = ["create", "tb_enable", "src_rcv", "steps", "destroy"]
    print("rep", rep, " ".join("%s %.4f" % (n, t[i + 1] - t[i]) for i, n in enumerate(names)),
          "total %.4f" % (t[-1] - t[0]), flush=True)
