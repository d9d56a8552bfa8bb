"""Where rafd_create (+ temporal blocking) spends its time on the C4 hall from
pinned host buffers (the e2e leg of bench.py): wall-clock per API call."""
import math
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd  # noqa: E402

cfg = bench.workload("C4", 1)
nx, ny, nz = cfg["room"]
beta0, D, E, F = I.config_materials(cfg)
dev = torch.device("cuda", 0)
mask_d, mm_d, _ = bench.slab_inputs(cfg, 0, nz, dev)
mask_h = torch.empty(mask_d.shape, dtype=torch.uint8, pin_memory=True)
mm_h = torch.empty(mm_d.shape, dtype=torch.uint8, pin_memory=True)
mask_h.copy_(mask_d)
mm_h.copy_(mm_d)
del mask_d, mm_d
torch.cuda.synchronize()
torch.cuda.empty_cache()
mm_dev = mm_h.to(dev) if len(sys.argv) > 1 and sys.argv[1] == "devmm" else None
for rep in range(3):
    t0 = time.perf_counter()
    room = rafd.Room(mask_h.numpy(), 1 / math.sqrt(3), 32, beta0, D, E, F,
                     matmap=mm_h.numpy() if mm_dev is None else mm_dev)
    t1 = time.perf_counter()
    room.set_temporal_blocking(2)
    t2 = time.perf_counter()
    room.set_source(I.source_position((nx, ny, nz)), I.impulse())
    room.set_receivers(I.receiver_positions((nx, ny, nz)))
    t3 = time.perf_counter()
    room.step(2)
    room.synchronize()
    t4 = time.perf_counter()
    room.destroy()
    t5 = time.perf_counter()
    print(f"rep {rep}: create {1e3*(t1-t0):.1f} ms, temporal blocking {1e3*(t2-t1):.1f} ms, "
          f"source+receivers {1e3*(t3-t2):.1f} ms, first double step {1e3*(t4-t3):.1f} ms, destroy {1e3*(t5-t4):.1f} ms")
