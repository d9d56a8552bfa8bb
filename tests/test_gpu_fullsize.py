"""Parity at BASELINE.json's full size, in the configuration bench.py times:
the C4 hall (1536x1024x704 = 1.107e9 voxels, FD-MM MB=3, M=8, fp32), default
volume-kernel tiling, inputs generated on the device exactly as bench.py does.
From a seeded random state (fields and branch state) both the CUDA path and
the oracle take 2 steps; every voxel, every branch state and the receivers are
compared bit for bit.  Host memory ~40 GB, ~1-2 min."""
import math

import numpy as np
import pytest
import torch

import bench
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from paper_conf_ipps_stoltzfushsld21_b200 import rafd

pytestmark = pytest.mark.gpu
LAM = 1.0 / math.sqrt(3.0)


def test_c4_full_size_two_steps_bitwise(orc):
    cfg = bench.workload("C4", 1)
    nx, ny, nz = cfg["room"]
    beta0, D, E, F = I.config_materials(cfg)
    dev = torch.device("cuda", 0)
    mask_d, mm_d, _ = bench.slab_inputs(cfg, 0, nz, dev)
    g = rafd.Room(mask_d, LAM, 32, beta0, D, E, F, matmap=mm_d)
    nb = g.nb
    gen = torch.Generator(device=dev).manual_seed(20251017)
    up = torch.rand((nz, ny, nx), generator=gen, device=dev, dtype=torch.float32) * 2 - 1
    uc = torch.rand((nz, ny, nx), generator=gen, device=dev, dtype=torch.float32) * 2 - 1
    v0 = (torch.rand((3, nb), generator=gen, device=dev, dtype=torch.float32) - 0.5) * 0.2
    g0 = (torch.rand((3, nb), generator=gen, device=dev, dtype=torch.float32) - 0.5) * 0.2
    g.set_state(up, uc, v0, g0)
    src = I.source_position((nx, ny, nz))
    rcv = I.receiver_positions((nx, ny, nz))
    g.set_source(src, [1.0, -0.5])
    g.set_receivers(rcv)
    g.step(2)

    o = orc.OracleRoom(mask_d.cpu().numpy(), LAM, 32, beta0, D, E, F, matmap=mm_d.cpu().numpy())
    del mask_d, mm_d
    assert o.nb == nb
    o.set_state(up.cpu().numpy(), uc.cpu().numpy(), v0.cpu().numpy(), g0.cpu().numpy())
    del up, uc
    o.set_source(src, [1.0, -0.5])
    o.set_receivers(rcv)
    o.step(2)

    cur_g = torch.empty((nz, ny, nx), dtype=torch.float32, device=dev)
    prv_g = torch.empty_like(cur_g)
    g.read_field(out_curr=cur_g, out_prev=prv_g)
    cur_o, prv_o = o.read_field()
    assert np.array_equal(cur_g.cpu().numpy(), cur_o)
    assert np.array_equal(prv_g.cpu().numpy(), prv_o)
    vg, gg = g.read_branch_state()
    vo, go = o.read_branch_state()
    assert np.array_equal(vg, vo) and np.array_equal(gg, go)
    assert np.array_equal(g.read_receivers(), o.read_receivers())
