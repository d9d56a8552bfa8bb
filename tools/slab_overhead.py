"""Cost of the z-slab machinery on one GPU: the C4 hall stepped whole vs as p
in-process slabs (rafd_step_group: edge phases, halo peer copies, interior
phases), temporal blocking on or off.  Wall clock around `steps` steps after a
warm-up, device synchronised on both sides (no profiling events)."""
import math
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd  # noqa: E402

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 40
cfg = bench.workload("C4", 1)
nx, ny, nz = cfg["room"]
beta0, D, E, F = I.config_materials(cfg)
dev = torch.device("cuda", 0)
mask, mm, _ = bench.slab_inputs(cfg, 0, nz, dev)
LAM = 1 / math.sqrt(3)
for tb in (2, 1):
    for p in (1, 2, 4):
        if p == 1:
            rooms = [rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)]
        else:
            plan = bench.slab_plan_box(nx, ny, nz, 32, 3, p)
            rooms = [rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=k, nranks=p, z_begin=a, z_end=b)
                     for k, (a, b) in enumerate(plan)]
        for r in rooms:
            r.set_temporal_blocking(tb)
            r.set_source(I.source_position((nx, ny, nz)), I.impulse())

        def run(n):
            if p == 1:
                rooms[0].step(n)
            else:
                rafd.rafd_step_group(rooms, n)
        run(4)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        run(steps)
        torch.cuda.synchronize()
        ms = (time.perf_counter() - t0) * 1e3 / steps
        print(f"tb {tb} slabs {p}: {ms:.3f} ms/step, {nx * ny * nz / ms / 1e6:.1f} Gvox/s", flush=True)
        for r in rooms:
            r.destroy()
        torch.cuda.empty_cache()
