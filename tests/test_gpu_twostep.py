"""GPU parity of temporal blocking (rafd_set_temporal_blocking(2): two leapfrog
steps per grid sweep, twostep.cu) against the CPU oracle, which takes single
steps exactly as Listings 2-4 describe.

The two-step path evaluates the same expressions in the same order, so the bar
is bitwise equality (the north_star tolerance is asserted too): fields, branch
state, receivers, after even and odd step counts, with the source in the
interior, on a boundary node and on a room-end plane, for ragged tile counts,
thin rooms and non-cuboid shapes; plus switching the mode mid-run, checkpoints
taken while the state lives in the second buffer pair, and graph replay.
"""
import json
import math
import os

import numpy as np
import pytest
import torch

from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from paper_conf_ipps_stoltzfushsld21_b200 import rafd

pytestmark = pytest.mark.gpu
LAM = 1.0 / math.sqrt(3.0)
TOL = {32: 1e-5, 64: 1e-12}
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module", autouse=True)
def _lib():
    from paper_conf_ipps_stoltzfushsld21_b200 import build
    build.build()
    assert torch.cuda.is_available()


@pytest.fixture(autouse=True)
def _two_kernel(monkeypatch):
    monkeypatch.setenv("RAFD_FUSED", "0")


def tb_room(mask, precision, beta0, D=None, E=None, F=None, matmap=None, lam=LAM):
    g = rafd.Room(mask, lam, precision, beta0, D, E, F, matmap=matmap)
    g.set_temporal_blocking(2)
    assert g.get_info()["steps_per_sweep"] == 2
    return g


def assert_same(a, b, precision, what):
    peak = max(np.abs(a).max(), 1e-300)
    err = np.abs(a.astype(np.float64) - b.astype(np.float64)).max()
    assert err <= TOL[precision] * peak, f"{what}: max|d| = {err:.3e} (peak {peak:.3e})"
    assert np.array_equal(a, b), f"{what}: within tolerance ({err:.3e}) but not bitwise"


def compare(o, g, precision, branches=False):
    co, po = o.read_field()
    cg, pg = g.read_field()
    assert_same(co, cg, precision, "u^n")
    assert_same(po, pg, precision, "u^{n-1}")
    ro, rg = o.read_receivers(), g.read_receivers()
    if ro.size or rg.size:
        assert_same(ro, rg, precision, "receivers")
    if branches:
        vo, go = o.read_branch_state()
        vg, gg = g.read_branch_state()
        assert_same(vo, vg, precision, "v")
        assert_same(go, gg, precision, "g")


@pytest.mark.parametrize("nsteps", [500, 499])
def test_c1_worked_example(orc, nsteps):
    """C1 (64^3 rigid box, fp64, impulse at (19,25,32), 8 receivers): the
    receiver traces equal the oracle's and the DCT-II golden values."""
    mask = I.box_mask(64, 64, 64).numpy()
    o = orc.OracleRoom(mask, LAM, 64, np.zeros(1))
    g = tb_room(mask, 64, np.zeros(1))
    rcv = I.receiver_positions((64, 64, 64))
    for r in (o, g):
        r.set_source((19, 25, 32), [1.0])
        r.set_receivers(rcv)
        r.step(nsteps)
    co, cg = o.read_field()[0], g.read_field()[0]
    assert_same(co, cg, 64, "u^n")
    ro, rg = o.read_receivers(), g.read_receivers()
    assert_same(ro, rg, 64, "receivers")
    gold = json.load(open(os.path.join(GOLDEN, "c1_receivers.json")))
    assert [list(p) for p in rcv] == gold["receivers_xyz"]
    for v in gold["values"]:
        if v["n"] < nsteps:
            assert abs(rg[v["receiver"], v["n"]] - v["value"]) <= 1e-12 * gold["peak_abs"]


@pytest.mark.parametrize("precision", [32, 64])
@pytest.mark.parametrize("MB", [0, 1, 3])
@pytest.mark.parametrize("shape", ["blob", "dome", "lshape"])
def test_random_state_bitwise(orc, precision, MB, shape):
    """Random fields and branch state, 5 random materials, a source, 301 steps
    (150 double steps + 1 single): fields, branch state, receivers bitwise."""
    dims = (131, 37, 19)  # 2 x-tiles (120 columns each) + ragged, 2 y-tiles (32 rows) + ragged
    mask = I.make_mask(shape, *dims, seed=MB).numpy() if shape != "blob" else \
        I.blob_mask(*dims, seed=MB, fill=0.8).numpy()
    mm = I.material_map(torch.from_numpy(mask), "random", 5).numpy()
    if MB:
        beta0, D, E, F = I.fd_tables(5, MB, seed=100 + MB)
        beta0 = np.array([0.0, 0.02, 0.0, 0.1, 0.3])
    else:
        beta0, D, E, F = np.array([0.0, 0.05, 0.2, 0.6, 0.9]), None, None, None
    o = orc.OracleRoom(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    g = tb_room(mask, precision, beta0, D, E, F, matmap=mm)
    dt = np.float32 if precision == 32 else np.float64
    rng = np.random.default_rng(MB + 10 * precision)
    up = rng.uniform(-1, 1, mask.shape).astype(dt)
    uc = rng.uniform(-1, 1, mask.shape).astype(dt)
    args = [up, uc]
    if MB:
        nb = o.nb
        args += [rng.uniform(-0.1, 0.1, (MB, nb)).astype(dt), rng.uniform(-0.1, 0.1, (MB, nb)).astype(dt)]
    src = I.snap_inside(mask, (60, 18, 9))
    rcv = [I.snap_inside(mask, p) for p in [(3, 3, 3), (61, 18, 9), (119, 31, 18), (120, 32, 10)]]
    for r in (o, g):
        r.set_state(*args)
        r.set_source(src, I.gaussian_pulse(50, 5.0))
        r.set_receivers(rcv)
        r.step(301)
    compare(o, g, precision, branches=MB > 0)
    eo, eg = o.energy(), g.energy()
    assert abs(eo - eg) <= 1e-9 * abs(eo)


@pytest.mark.parametrize("where", ["wall", "floor_plane", "next_to_wall", "corner"])
@pytest.mark.parametrize("precision,MB", [(32, 3), (64, 0)])
def test_source_positions(orc, where, precision, MB):
    """The source on a boundary node, on the first plane, beside a wall and in
    a corner: its 7-point star is recomputed after the injection."""
    mask = I.lshape_mask(70, 40, 12).numpy()
    mm = I.material_map(torch.from_numpy(mask), "random", 4).numpy()
    if MB:
        beta0, D, E, F = I.fd_tables(4, MB, seed=7)
    else:
        beta0, D, E, F = np.array([0.05, 0.2, 0.6, 0.9]), None, None, None
    o = orc.OracleRoom(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    g = tb_room(mask, precision, beta0, D, E, F, matmap=mm)
    K = o.classification()[0]
    if where == "wall":
        z, y, x = np.argwhere((K > 0) & (K < 6))[400]
    elif where == "floor_plane":
        z, y, x = 0, 20, 30
    elif where == "next_to_wall":
        z, y, x = 6, 1, 33
    else:
        z, y, x = 0, 0, 0
    src = (int(x), int(y), int(z))
    assert K[src[2], src[1], src[0]] > 0
    for r in (o, g):
        r.set_source(src, I.gaussian_pulse(80, 6.0))
        r.set_receivers([src, I.snap_inside(mask, (min(int(x) + 1, 69), int(y), int(z))), (5, 5, 5)])
        r.step(121)
    compare(o, g, precision, branches=MB > 0)


@pytest.mark.parametrize("dims", [(1, 1, 1), (1, 1, 40), (300, 1, 1), (1, 50, 3), (120, 32, 2), (121, 33, 3),
                                  (239, 65, 5), (2, 2, 2)])
@pytest.mark.parametrize("precision", [32, 64])
def test_thin_and_ragged_rooms(orc, dims, precision):
    """Degenerate and tile-edge room sizes (x multiples of 120 / 60 columns and
    y multiples of 32 rows, plus one) with FI walls, from a random state."""
    mask = np.ones(dims[::-1], np.uint8)
    beta0 = np.array([0.3])
    o = orc.OracleRoom(mask, LAM, precision, beta0)
    g = tb_room(mask, precision, beta0)
    dt = np.float32 if precision == 32 else np.float64
    rng = np.random.default_rng(sum(dims))
    up = rng.uniform(-1, 1, mask.shape).astype(dt)
    uc = rng.uniform(-1, 1, mask.shape).astype(dt)
    src = (dims[0] // 2, dims[1] // 2, dims[2] // 2)
    inside = o.classification()[0][src[2], src[1], src[0]] > 0  # a 1x1x1 room's voxel is isolated (K = 0)
    for r in (o, g):
        r.set_state(up, uc)
        if inside:
            r.set_source(src, [1.0, -0.5])
            r.set_receivers([src])
        r.step(37)
    compare(o, g, precision)


def test_mode_switching_and_checkpoint(orc):
    """1 -> 2 -> 1 -> 2 steps per sweep mid-run, a checkpoint read while the
    state lives in the second buffer pair and restored into a fresh room."""
    mask = I.dome_mask(90, 70, 30).numpy()
    mm = I.material_map(torch.from_numpy(mask), "random", 3).numpy()
    beta0, D, E, F = I.fd_tables(3, 2, seed=3)
    o = orc.OracleRoom(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    g = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    for r in (o, g):
        r.set_source((45, 35, 10), I.gaussian_pulse(60, 5.0))
        r.set_receivers([(45, 35, 10), (20, 30, 20)])
    o.step(7)
    g.step(7)
    g.set_temporal_blocking(2)
    o.step(10)
    g.step(10)  # state now in the second pair
    g.set_temporal_blocking(1)
    o.step(3)
    g.step(3)
    g.set_temporal_blocking(2)
    o.step(20)
    g.step(20)
    compare(o, g, 32, branches=True)
    # checkpoint from the two-step room, resume in a fresh two-step room
    cur, prev = g.read_field()
    v, gs = g.read_branch_state()
    n = g.get_info()["steps"]
    h = tb_room(mask, 32, beta0, D, E, F, matmap=mm)
    h.set_source((45, 35, 10), I.gaussian_pulse(60, 5.0))
    h.set_receivers([(45, 35, 10), (20, 30, 20)])
    h.set_state(prev, cur, v, gs)
    h.set_step(n)
    o.step(33)
    h.step(33)
    compare(o, h, 32, branches=True)


def test_graph_direct_and_single_step_agree(orc):
    """CUDA-graph replay of double steps, one-by-one launches with profiling,
    and the single-step path give identical bits; launch accounting."""
    mask = I.dome_mask(40, 40, 40).numpy()
    beta0, D, E, F = I.fd_tables(2, 3)
    mm = I.material_map(torch.from_numpy(mask), "random", 2).numpy()
    a = tb_room(mask, 32, beta0, D, E, F, matmap=mm)
    b = tb_room(mask, 32, beta0, D, E, F, matmap=mm)
    c = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    for r in (a, b, c):
        r.set_source((20, 20, 10), [1.0])
    a.step(67)
    b.set_profiling(True)
    for _ in range(33):
        b.step(2)
    b.step(1)
    c.step(67)
    t = b.get_kernel_times()
    # per double step: k_volume2, the step-(n+1) boundary kernel (+ source/receivers
    # in its last block), and the shell fused with the step-(n+2) boundary update
    # (+ source/receivers); the odd step: volume + boundary
    assert t["volume_launches"] == 34 and t["shell_launches"] == 33 and t["boundary_launches"] == 34
    assert np.array_equal(a.read_field()[0], b.read_field()[0])
    assert np.array_equal(a.read_field()[0], c.read_field()[0])
    assert a.launch_count() == b.launch_count() == 33 * 3 + 2


def test_errors():
    mask = I.box_mask(20, 20, 20).numpy()
    g = rafd.Room(mask, LAM, 32, np.array([0.1]))
    with pytest.raises(rafd.RafdError):
        g.set_temporal_blocking(3)
    s = rafd.Room(mask, LAM, 32, np.array([0.1]), scheme=1)
    with pytest.raises(rafd.RafdError):
        s.set_temporal_blocking(2)
    with pytest.raises(rafd.RafdError):  # the halo push needs an IPC-connected slab
        g.set_halo_push(True)
    g.set_halo_push(False)


@pytest.mark.parametrize("precision,MB,shape,dims", [(32, 0, "lshape", (96, 88, 80)), (32, 3, "dome", (90, 84, 76)),
                                                   (64, 3, "box", (70, 64, 60))])
def test_long_run_1000_steps(orc, precision, MB, shape, dims):
    """The north_star tolerance is stated after 1000 steps: an impulse response
    of 1000 steps (graph replays of 16 steps plus direct double steps) with
    temporal blocking, FI-MM on an L-shape and FD-MM on a dome / box, against
    the oracle's single steps -- bitwise."""
    mask_t = I.make_mask(shape, *dims)
    M = 4 if MB == 0 else 8
    mm = I.material_map(mask_t, "region", M).numpy()
    mask = mask_t.numpy()
    if MB:
        beta0, D, E, F = I.fd_tables(M, MB)
    else:
        beta0, D, E, F = I.fi_beta_from_alpha([0.05, 0.2, 0.5, 0.9]), None, None, None
    src = I.source_position(dims, mask)
    rcv = I.receiver_positions(dims, mask)
    o = orc.OracleRoom(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    g = tb_room(mask, precision, beta0, D, E, F, matmap=mm)
    for r in (o, g):
        r.set_source(src, I.impulse())
        r.set_receivers(rcv)
    o.step(1000)
    g.step(998)
    g.step(2)
    compare(o, g, precision, branches=bool(MB))
