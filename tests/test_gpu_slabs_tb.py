"""Temporal blocking in z slabs (SURVEY §8(e) x §8(f) f4): every slab runs the
double step edge planes first -- u^{n+1} of its first / last owned plane with
the single-step kernel (Listing 2 + Listings 3/4, PAPER.md:349-357, 371-377,
415-440), exchanged while the two-step kernel advances the interior planes,
then u^{n+2} of the edge planes from the exchanged u^{n+1} -- and must
reproduce the undivided room (single steps) and the oracle bit for bit."""
import math

import numpy as np
import pytest
import torch

from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from paper_conf_ipps_stoltzfushsld21_b200 import rafd

pytestmark = pytest.mark.gpu
LAM = 1.0 / math.sqrt(3.0)


@pytest.fixture(autouse=True)
def two_kernel(monkeypatch):
    monkeypatch.setenv("RAFD_FUSED", "0")


def make_case(shape, dims, MB, M, seed):
    nx, ny, nz = dims
    mask_t = I.make_mask(shape, nx, ny, nz, seed=seed)
    mm = I.material_map(mask_t, "region" if M in (4, 8) else "random", M).numpy()
    mask = mask_t.numpy()
    if MB:
        beta0, D, E, F = I.fd_tables(M, MB, seed=seed)
    else:
        beta0, D, E, F = I.fi_beta_from_alpha(np.linspace(0.1, 0.8, M)), None, None, None
    return mask, mm, beta0, D, E, F


@pytest.mark.parametrize("p", [2, 3, 5])
@pytest.mark.parametrize("precision,MB,shape", [(32, 3, "dome"), (64, 2, "blob"), (32, 0, "lshape")])
def test_tb_slabs_equal_single_room(orc, p, precision, MB, shape):
    dims = (45, 38, 31)
    mask, mm, beta0, D, E, F = make_case(shape, dims, MB, 8, seed=p)
    dt = np.float32 if precision == 32 else np.float64
    rng = np.random.default_rng(p)
    up = rng.uniform(-1, 1, mask.shape).astype(dt)
    uc = rng.uniform(-1, 1, mask.shape).astype(dt)
    src = I.source_position(dims, mask)
    rcv = I.receiver_positions(dims, mask)
    sig = I.gaussian_pulse(40, 4.0)

    whole = rafd.Room(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    nb = whole.nb
    v0 = rng.uniform(-0.1, 0.1, (MB, nb)).astype(dt)
    g0 = rng.uniform(-0.1, 0.1, (MB, nb)).astype(dt)
    whole.set_state(up, uc, v0 if MB else None, g0 if MB else None)
    whole.set_source(src, sig)
    whole.set_receivers(rcv)

    plan = rafd.rafd_slab_plan(mask, precision, MB, p)
    slabs = [rafd.Room(mask, LAM, precision, beta0, D, E, F, matmap=mm, rank=k, nranks=p,
                       z_begin=a, z_end=b) for k, (a, b) in enumerate(plan)]
    off = 0
    for s in slabs:
        n = s.nb
        s.set_temporal_blocking(2)
        s.set_state(up, uc, v0[:, off:off + n] if MB else None, g0[:, off:off + n] if MB else None)
        off += n
        s.set_source(src, sig)
        s.set_receivers(rcv)
    assert off == nb
    assert all(s.get_info()["steps_per_sweep"] == 2 for s in slabs)

    whole.step(120)
    rafd.rafd_step_group(slabs, 77)   # 38 double steps + 1 single
    rafd.rafd_step_group(slabs, 43)

    cw, pw = whole.read_field()
    cs = np.concatenate([s.read_field()[0] for s in slabs])
    ps = np.concatenate([s.read_field()[1] for s in slabs])
    assert np.array_equal(cw, cs)
    assert np.array_equal(pw, ps)
    if MB:
        vw, gw = whole.read_branch_state()
        vs = np.concatenate([s.read_branch_state()[0] for s in slabs], axis=1)
        gs = np.concatenate([s.read_branch_state()[1] for s in slabs], axis=1)
        assert np.array_equal(vw, vs) and np.array_equal(gw, gs)
    rw = whole.read_receivers()
    rs = rafd.gather_receivers([s.read_receivers() for s in slabs], rcv, plan)
    assert np.array_equal(rw, rs)
    o = orc.OracleRoom(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    o.set_state(up, uc, v0 if MB else None, g0 if MB else None)
    o.set_source(src, sig)
    o.step(120)
    assert np.array_equal(o.read_field()[0], cs)


@pytest.mark.parametrize("where", ["first", "last", "interior", "second"])
def test_tb_thin_slabs_source_on_edges(where):
    """Slabs of 1, 2, 3, 4 and 5 planes (no interior, or one interior plane);
    the source on an edge plane, an interior plane, or the plane next to an
    edge (its star reaches the edge plane the exchange provides)."""
    dims = (30, 26, 15)
    mask, mm, beta0, D, E, F = make_case("box", dims, 3, 8, seed=4)
    plan = [(0, 1), (1, 3), (3, 6), (6, 10), (10, 15)]
    z = {"first": 3, "last": 9, "interior": 8, "second": 11}[where]
    src = (12, 11, z)
    rcv = [(5, 5, 0), (7, 8, 1), (8, 9, 2), (9, 9, 3), (10, 10, 6), (11, 11, 7), (12, 12, 11), (3, 4, 14)]
    whole = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    slabs = [rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=k, nranks=len(plan), z_begin=a, z_end=b)
             for k, (a, b) in enumerate(plan)]
    for r in [whole] + slabs:
        if r is not whole:
            r.set_temporal_blocking(2)
        r.set_source(src, I.gaussian_pulse(16, 2.0))
        r.set_receivers(rcv)
    whole.step(51)
    rafd.rafd_step_group(slabs, 51)
    cw, pw = whole.read_field()
    assert np.array_equal(cw, np.concatenate([s.read_field()[0] for s in slabs]))
    assert np.array_equal(pw, np.concatenate([s.read_field()[1] for s in slabs]))
    rw = whole.read_receivers()
    rs = rafd.gather_receivers([s.read_receivers() for s in slabs], rcv, plan)
    assert np.array_equal(rw, rs) and np.abs(rw).max() > 0


def test_tb_c4_section_slabs_bitwise():
    """A 64-plane section of the C4 hall (full 1536 x 1024 x-y section) as 4
    slabs with temporal blocking vs the whole room with temporal blocking: the
    bench's multi-GPU geometry at full x-y size."""
    nx, ny, nz = 1536, 1024, 64
    mask = torch.ones((nz, ny, nx), dtype=torch.uint8, device="cuda")
    mm = I.region_map_box(nx, ny, nz, 0, nz, device="cuda")
    beta0, D, E, F = I.fd_tables(8, 3)
    whole = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    whole.set_temporal_blocking(2)
    plan = [(0, 16), (16, 33), (33, 48), (48, 64)]
    slabs = [rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=k, nranks=4, z_begin=a, z_end=b)
             for k, (a, b) in enumerate(plan)]
    src = (700, 500, 32)
    for r in [whole] + slabs:
        if r is not whole:
            r.set_temporal_blocking(2)
        r.set_source(src, I.gaussian_pulse(20, 3.0))
    whole.step(60)
    rafd.rafd_step_group(slabs, 60)
    fw = torch.empty((nz, ny, nx), dtype=torch.float32, device="cuda")
    pw = torch.empty_like(fw)
    whole.read_field(out_curr=fw, out_prev=pw)
    for s, (a, b) in zip(slabs, plan):
        fs = torch.empty((b - a, ny, nx), dtype=torch.float32, device="cuda")
        ps = torch.empty_like(fs)
        s.read_field(out_curr=fs, out_prev=ps)
        assert torch.equal(fs, fw[a:b]) and torch.equal(ps, pw[a:b])
    assert float(fw.abs().max()) > 1e-4


def test_tb_group_mixed_settings_rejected():
    dims = (20, 18, 12)
    mask, mm, beta0, D, E, F = make_case("box", dims, 0, 4, seed=1)
    plan = [(0, 6), (6, 12)]
    slabs = [rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=k, nranks=2, z_begin=a, z_end=b)
             for k, (a, b) in enumerate(plan)]
    slabs[0].set_temporal_blocking(2)
    with pytest.raises(rafd.RafdError) as e:
        rafd.rafd_step_group(slabs, 4)
    assert e.value.code == rafd.RAFD_E_STATE


def test_tb_slabs_mode_switching_and_checkpoint(orc):
    """Slabs switching 1 -> 2 -> 1 -> 2 steps per sweep mid-run (the state
    moves between buffer pairs), then a checkpoint of every slab restored into
    fresh slabs with a different z split: equal to the oracle throughout."""
    dims = (50, 40, 23)
    mask, mm, beta0, D, E, F = make_case("dome", dims, 2, 3, seed=7)
    src = (25, 20, 7)
    rcv = [(25, 20, 7), (10, 15, 15), (30, 25, 2)]
    sig = I.gaussian_pulse(50, 4.0)
    o = orc.OracleRoom(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    o.set_source(src, sig)
    o.set_receivers(rcv)

    def make(plan):
        ss = [rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=k, nranks=len(plan), z_begin=a, z_end=b)
              for k, (a, b) in enumerate(plan)]
        for s in ss:
            s.set_source(src, sig)
            s.set_receivers(rcv)
        return ss

    plan = [(0, 6), (6, 8), (8, 16), (16, 23)]
    slabs = make(plan)
    for n, tb in ((7, 1), (10, 2), (3, 1), (21, 2)):
        for s in slabs:
            s.set_temporal_blocking(tb)
        rafd.rafd_step_group(slabs, n)
        o.step(n)
        assert np.array_equal(o.read_field()[0], np.concatenate([s.read_field()[0] for s in slabs]))
    rs = rafd.gather_receivers([s.read_receivers() for s in slabs], rcv, plan)
    assert np.array_equal(o.read_receivers().astype(np.float32), rs.astype(np.float32))
    # checkpoint every slab, restore into a different split (temporal blocking on)
    cur = np.concatenate([s.read_field()[0] for s in slabs])
    prv = np.concatenate([s.read_field()[1] for s in slabs])
    v = np.concatenate([s.read_branch_state()[0] for s in slabs], axis=1)
    g = np.concatenate([s.read_branch_state()[1] for s in slabs], axis=1)
    nsteps = slabs[0].get_info()["steps"]
    plan2 = [(0, 11), (11, 12), (12, 23)]
    slabs2 = make(plan2)
    off = 0
    for s in slabs2:
        s.set_temporal_blocking(2)
        n = s.nb
        s.set_state(prv, cur, v[:, off:off + n], g[:, off:off + n])
        s.set_step(nsteps)
        off += n
    rafd.rafd_step_group(slabs2, 33)
    o.step(33)
    assert np.array_equal(o.read_field()[0], np.concatenate([s.read_field()[0] for s in slabs2]))
    assert np.array_equal(o.read_field()[1], np.concatenate([s.read_field()[1] for s in slabs2]))
