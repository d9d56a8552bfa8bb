"""Parity at BASELINE.json's full size, in the configuration bench.py times:
the C4 hall (1536x1024x704 = 1.107e9 voxels, FD-MM MB=3, M=8, fp32), default
volume-kernel tiling, inputs generated on the device exactly as bench.py does.
From a seeded random state (fields and branch state) both the CUDA path and
the oracle take 2 steps -- the CUDA path once with single steps and once with
temporal blocking (one double step of k_volume2 + shell, the bench default) --
and every voxel, every branch state and the receivers are compared bit for
bit.  Host memory ~40 GB, ~1-2 min."""
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
    g2 = rafd.Room(mask_d, LAM, 32, beta0, D, E, F, matmap=mm_d)
    g2.set_temporal_blocking(2)
    nb = g.nb
    gen = torch.Generator(device=dev).manual_seed(20251017)
    up = torch.rand((nz, ny, nx), generator=gen, device=dev, dtype=torch.float32) * 2 - 1
    uc = torch.rand((nz, ny, nx), generator=gen, device=dev, dtype=torch.float32) * 2 - 1
    v0 = (torch.rand((3, nb), generator=gen, device=dev, dtype=torch.float32) - 0.5) * 0.2
    g0 = (torch.rand((3, nb), generator=gen, device=dev, dtype=torch.float32) - 0.5) * 0.2
    src = I.source_position((nx, ny, nz))
    rcv = I.receiver_positions((nx, ny, nz))
    for r in (g, g2):
        r.set_state(up, uc, v0, g0)
        r.set_source(src, [1.0, -0.5])
        r.set_receivers(rcv)
        r.step(2)

    o = orc.OracleRoom(mask_d.cpu().numpy(), LAM, 32, beta0, D, E, F, matmap=mm_d.cpu().numpy())
    del mask_d, mm_d
    assert o.nb == nb
    o.set_state(up.cpu().numpy(), uc.cpu().numpy(), v0.cpu().numpy(), g0.cpu().numpy())
    del up, uc
    o.set_source(src, [1.0, -0.5])
    o.set_receivers(rcv)
    o.step(2)

    cur_o, prv_o = o.read_field()
    vo, go = o.read_branch_state()
    rec_o = o.read_receivers()
    for r in (g, g2):
        cur_g = torch.empty((nz, ny, nx), dtype=torch.float32, device=dev)
        prv_g = torch.empty_like(cur_g)
        r.read_field(out_curr=cur_g, out_prev=prv_g)
        assert np.array_equal(cur_g.cpu().numpy(), cur_o)
        assert np.array_equal(prv_g.cpu().numpy(), prv_o)
        del cur_g, prv_g
        vg, gg = r.read_branch_state()
        assert np.array_equal(vg, vo) and np.array_equal(gg, go)
        assert np.array_equal(r.read_receivers(), rec_o)


def test_c4_full_size_many_steps_bitwise(orc):
    """The bench configuration over many launches: C4 with temporal blocking,
    37 steps in one rafd_step call (two 16-step CUDA graphs of double steps,
    then two double steps and a single step), so the dynamic unit counter of
    k_volume2 is reset and reused across 18 launches and the graph and direct
    paths hand the state to each other.  Every voxel, the branch state and
    the receivers bitwise against the oracle (the oracle runs on all host
    cores)."""
    cfg = bench.workload("C4", 1)
    nx, ny, nz = cfg["room"]
    beta0, D, E, F = I.config_materials(cfg)
    dev = torch.device("cuda", 0)
    mask_d, mm_d, _ = bench.slab_inputs(cfg, 0, nz, dev)
    g = rafd.Room(mask_d, LAM, 32, beta0, D, E, F, matmap=mm_d)
    g.set_temporal_blocking(2)
    gen = torch.Generator(device=dev).manual_seed(37)
    up = torch.rand((nz, ny, nx), generator=gen, device=dev, dtype=torch.float32) * 2 - 1
    uc = torch.rand((nz, ny, nx), generator=gen, device=dev, dtype=torch.float32) * 2 - 1
    src = I.source_position((nx, ny, nz))
    rcv = I.receiver_positions((nx, ny, nz))
    sig = I.gaussian_pulse(24, 4.0)
    g.set_state(up, uc)
    g.set_source(src, sig)
    g.set_receivers(rcv)
    g.step(37)
    o = orc.OracleRoom(mask_d.cpu().numpy(), LAM, 32, beta0, D, E, F, matmap=mm_d.cpu().numpy())
    del mask_d, mm_d
    o.set_state(up.cpu().numpy(), uc.cpu().numpy())
    del up, uc
    o.set_source(src, sig)
    o.set_receivers(rcv)
    o.step(37)
    cur_o, prv_o = o.read_field()
    cur_g = torch.empty((nz, ny, nx), dtype=torch.float32, device=dev)
    prv_g = torch.empty_like(cur_g)
    g.read_field(out_curr=cur_g, out_prev=prv_g)
    assert np.array_equal(cur_g.cpu().numpy(), cur_o)
    assert np.array_equal(prv_g.cpu().numpy(), prv_o)
    del cur_g, prv_g
    vg, gg = g.read_branch_state()
    vo, go = o.read_branch_state()
    assert np.array_equal(vg, vo) and np.array_equal(gg, go)
    assert np.array_equal(g.read_receivers(), o.read_receivers())


@pytest.mark.parametrize("name,precision,steps", [("C2a", 32, 30), ("C2b", 32, 30), ("C3", 32, 12), ("C3d", 64, 12)])
def test_config_full_size_bitwise(orc, name, precision, steps):
    """BASELINE.json configs[1..2] at full size (256^3 L-shape and dome with
    FI-MM M=4; 512x384x256 box with FD-MM MB=3 M=8 in fp32 and fp64): a few
    steps from a seeded random state plus the config's source, every voxel and
    the receivers bitwise -- with single steps and with temporal blocking."""
    cfg = I.CONFIGS[name]
    nx, ny, nz = cfg["dims"]
    mask_t = I.make_mask(cfg["shape"], nx, ny, nz)
    mm = I.material_map(mask_t, cfg["rule"], cfg["M"]).numpy()
    mask = mask_t.numpy()
    beta0, D, E, F = I.config_materials(cfg)
    g = rafd.Room(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    g2 = rafd.Room(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    g2.set_temporal_blocking(2)
    o = orc.OracleRoom(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    dt = np.float32 if precision == 32 else np.float64
    rng = np.random.default_rng(7)
    up = rng.uniform(-1, 1, mask.shape).astype(dt)
    uc = rng.uniform(-1, 1, mask.shape).astype(dt)
    src = I.source_position(cfg["dims"], mask)
    rcv = I.receiver_positions(cfg["dims"], mask)
    for r in (g, g2, o):
        r.set_state(up, uc)
        r.set_source(src, I.impulse())
        r.set_receivers(rcv)
        r.step(steps + 1)  # odd: the two-step room ends with one single step
    fo = o.read_field()[0]
    assert np.array_equal(g.read_field()[0], fo)
    assert np.array_equal(g2.read_field()[0], fo)
    ro = o.read_receivers()
    assert np.array_equal(g.read_receivers(), ro)
    assert np.array_equal(g2.read_receivers(), ro)
    if cfg["MB"]:
        vo, go = o.read_branch_state()
        for r in (g, g2):
            vg, gg = r.read_branch_state()
            assert np.array_equal(vg, vo) and np.array_equal(gg, go)


def test_c5_hall_int64_indexing_light_cone():
    """The C5 hall (2048x1536x2560 = 8.05e9 voxels, fp32, FD-MM) on one GPU:
    more than 2^32 grid elements, so boundary positions are int64.  A source
    next to the corner (10,10,10): after 50 steps the disturbance lies within
    50 voxels of it, so the C5 field must equal, bit for bit, that of a small
    box with the same corner walls (its far walls are beyond the light cone)."""
    cfg = bench.workload("C5", 1)
    nx, ny, nz = cfg["room"]
    beta0, D, E, F = I.config_materials(cfg)
    dev = torch.device("cuda", 0)
    mask, mm, _ = bench.slab_inputs(cfg, 0, nz, dev)
    big = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    del mask, mm
    torch.cuda.empty_cache()
    assert big.get_info()["n_boundary"] == 24616968
    src, steps, n = (10, 10, 10), 50, 128
    sig = I.gaussian_pulse(24, 3.0)
    big.set_source(src, sig)
    big.step(steps)
    cur = torch.empty((nz, ny, nx), dtype=torch.float32, device=dev)
    big.read_field(out_curr=cur, out_prev=False)
    corner = cur[:n, :n, :n].cpu().numpy()
    del cur, big
    torch.cuda.empty_cache()
    # the small box: same corner walls and, near the corner, the same region materials
    small_mask = np.ones((n, n, n), np.uint8)
    small_mm = I.region_map_box(nx, ny, nz, 0, n, device="cpu")[:, :n, :n].contiguous().numpy()
    small = rafd.Room(small_mask, LAM, 32, beta0, D, E, F, matmap=small_mm)
    small.set_source(src, sig)
    small.step(steps)
    ref = small.read_field()[0]
    reach = 10 + steps + 1
    assert np.array_equal(corner[:reach, :reach, :reach], ref[:reach, :reach, :reach])
    assert np.abs(ref).max() > 1e-3 and not np.any(corner[reach:, :, :])
