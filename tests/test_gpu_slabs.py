"""z-slab decomposition on one GPU ("virtual ranks"): p slab
handles of one room stepped with rafd_step_group (ghost planes exchanged by
device copies each step) must reproduce the undivided room bit for bit --
fields, branch state, receivers, classification -- and the oracle."""
import math

import numpy as np
import pytest
import torch

from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from paper_conf_ipps_stoltzfushsld21_b200 import rafd

pytestmark = pytest.mark.gpu
LAM = 1.0 / math.sqrt(3.0)


@pytest.fixture(autouse=True, params=["fused", "two-kernel"])
def step_form(request, monkeypatch):
    monkeypatch.setenv("RAFD_FUSED", "1" if request.param == "fused" else "0")
    return request.param


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
@pytest.mark.parametrize("precision,MB", [(32, 3), (64, 2), (32, 0)])
def test_slabs_equal_single_room(orc, p, precision, MB):
    dims = (45, 38, 31)
    mask, mm, beta0, D, E, F = make_case("dome", dims, MB, 8, seed=p)
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
    with pytest.raises(rafd.RafdError) as e:
        slabs[0].step(1)
    assert e.value.code == rafd.RAFD_E_STATE
    off = 0
    for s in slabs:
        n = s.nb
        s.set_state(up, uc, v0[:, off:off + n] if MB else None, g0[:, off:off + n] if MB else None)
        off += n
        s.set_source(src, sig)
        s.set_receivers(rcv)
    assert off == nb

    whole.step(120)
    rafd.rafd_step_group(slabs, 77)
    rafd.rafd_step_group(slabs, 43)

    cw, pw = whole.read_field()
    cs = np.concatenate([s.read_field()[0] for s in slabs])
    ps = np.concatenate([s.read_field()[1] for s in slabs])
    assert np.array_equal(cw, cs)
    assert np.array_equal(pw, ps)
    Kw, bw, kbw, mw = whole.get_classification()
    parts = [s.get_classification() for s in slabs]
    assert np.array_equal(Kw, np.concatenate([q[0] for q in parts]))
    for i in (1, 2, 3):
        assert np.array_equal([bw, kbw, mw][i - 1], np.concatenate([q[i] for q in parts]))
    if MB:
        vw, gw = whole.read_branch_state()
        vs = np.concatenate([s.read_branch_state()[0] for s in slabs], axis=1)
        gs = np.concatenate([s.read_branch_state()[1] for s in slabs], axis=1)
        assert np.array_equal(vw, vs) and np.array_equal(gw, gs)
    rw = whole.read_receivers()
    rs = rafd.gather_receivers([s.read_receivers() for s in slabs], rcv, plan)
    assert np.array_equal(rw, rs)
    ew = whole.energy()
    es = sum(s.energy() for s in slabs)
    assert abs(ew - es) <= 1e-9 * abs(ew)
    # and the oracle
    o = orc.OracleRoom(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    o.set_state(up, uc, v0 if MB else None, g0 if MB else None)
    o.set_source(src, sig)
    o.step(120)
    assert np.array_equal(o.read_field()[0], cs)


def test_c4_section_slabs_bitwise():
    """A thin section of the C4 hall (full x-y section, 64 planes) as 4 slabs
    vs the whole: the bench's multi-GPU geometry at full x-y size."""
    nx, ny, nz = 1536, 1024, 64
    mask = torch.ones((nz, ny, nx), dtype=torch.uint8, device="cuda")
    mm = I.region_map_box(nx, ny, nz, 0, nz, device="cuda")
    beta0, D, E, F = I.fd_tables(8, 3)
    whole = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    plan = [(0, 16), (16, 33), (33, 48), (48, 64)]
    slabs = [rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=k, nranks=4, z_begin=a, z_end=b)
             for k, (a, b) in enumerate(plan)]
    src = (700, 500, 31)
    for r in [whole] + slabs:
        r.set_source(src, I.gaussian_pulse(20, 3.0))
    whole.step(60)
    rafd.rafd_step_group(slabs, 60)
    fw = torch.empty((nz, ny, nx), dtype=torch.float32, device="cuda")
    whole.read_field(out_curr=fw, out_prev=torch.empty_like(fw))
    for s, (a, b) in zip(slabs, plan):
        fs = torch.empty((b - a, ny, nx), dtype=torch.float32, device="cuda")
        s.read_field(out_curr=fs, out_prev=torch.empty_like(fs))
        assert torch.equal(fs, fw[a:b])
    assert float(fw.abs().max()) > 1e-4


@pytest.mark.parametrize("where", ["first", "last", "interior"])
def test_slab_source_and_receivers_on_edge_planes(where):
    """Source / receivers on the planes handled by the edge phase (before the
    halo exchange) and on interior planes; thin slabs (1 and 2 planes) too."""
    dims = (30, 26, 12)
    mask, mm, beta0, D, E, F = make_case("box", dims, 3, 8, seed=4)
    plan = [(0, 1), (1, 3), (3, 7), (7, 12)]
    z = {"first": 3, "last": 6, "interior": 5}[where]
    src = (12, 11, z)
    rcv = [(5, 5, 0), (7, 8, 1), (8, 9, 2), (9, 9, 3), (10, 10, 6), (11, 11, 7), (12, 12, 11), (3, 4, 5)]
    whole = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    slabs = [rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=k, nranks=4, z_begin=a, z_end=b)
             for k, (a, b) in enumerate(plan)]
    for r in [whole] + slabs:
        r.set_source(src, I.gaussian_pulse(16, 2.0))
        r.set_receivers(rcv)
    whole.step(50)
    rafd.rafd_step_group(slabs, 50)
    cw = whole.read_field()[0]
    cs = np.concatenate([s.read_field()[0] for s in slabs])
    assert np.array_equal(cw, cs)
    rw = whole.read_receivers()
    rs = rafd.gather_receivers([s.read_receivers() for s in slabs], rcv, plan)
    assert np.array_equal(rw, rs) and np.abs(rw).max() > 0
