"""GPU parity: the CUDA path (librafd.so through the C-ABI) vs the CPU oracle on
identical seeded rooms, materials, sources and states.

Bar: classification (K, boundary list, K_b, mat_b) bit-exact; fields,
receivers and branch state bitwise equal (the arithmetic spec, DESIGN.md §4,
makes this reachable), and in any case within the north_star tolerance
(max |delta| <= 1e-5 of the peak in fp32, 1e-12 in fp64).
"""
import math

import numpy as np
import pytest
import torch

from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from paper_conf_ipps_stoltzfushsld21_b200 import rafd

pytestmark = pytest.mark.gpu
LAM = 1.0 / math.sqrt(3.0)
TOL = {32: 1e-5, 64: 1e-12}


@pytest.fixture(scope="module", autouse=True)
def _lib():
    from paper_conf_ipps_stoltzfushsld21_b200 import build
    build.build()
    assert torch.cuda.is_available()


@pytest.fixture(autouse=True, params=["fused", "two-kernel"])
def step_form(request, monkeypatch):
    """Every parity test runs with the boundary update fused into the volume
    kernel (default) and with the paper's two-kernel form (RAFD_FUSED=0)."""
    monkeypatch.setenv("RAFD_FUSED", "1" if request.param == "fused" else "0")
    return request.param


def pair(orc, mask, precision, beta0, D=None, E=None, F=None, matmap=None, lam=LAM, **kw):
    o = orc.OracleRoom(mask, lam, precision, beta0, D, E, F, matmap=matmap)
    g = rafd.Room(mask, lam, precision, beta0, D, E, F, matmap=matmap, **kw)
    return o, g


def assert_close(a, b, precision, what):
    peak = max(np.abs(a).max(), 1e-300)
    err = np.abs(a.astype(np.float64) - b.astype(np.float64)).max()
    assert err <= TOL[precision] * peak, f"{what}: max|d| = {err:.3e} (peak {peak:.3e})"
    assert np.array_equal(a, b), f"{what}: within tolerance ({err:.3e}) but not bitwise"


def check_classification(o, g):
    Ko, bo, kbo, mo = o.classification()
    Kg, bg, kbg, mg = g.get_classification()
    assert np.array_equal(Ko, Kg)
    assert np.array_equal(bo, bg)
    assert np.array_equal(kbo, kbg)
    assert np.array_equal(mo, mg)
    io, ig = o.info(), g.get_info()
    for k in ("n_mask", "n_inside", "n_boundary", "isolated"):
        assert io[k] == ig[k], k
    assert list(io["k_hist"]) == list(ig["k_hist"])


ROOMS = {
    "box_ragged": lambda: I.box_mask(37, 23, 19).numpy(),
    "lshape": lambda: I.lshape_mask(40, 36, 20).numpy(),
    "dome": lambda: I.dome_mask(44, 40, 36).numpy(),
    "blob": lambda: I.blob_mask(33, 29, 17, seed=8, fill=0.75).numpy(),
    "duct": lambda: np.ones((1, 1, 300), np.uint8),
    "slab1": lambda: np.ones((1, 17, 29), np.uint8),
}


@pytest.mark.parametrize("room", list(ROOMS))
def test_classification_bit_exact(orc, room):
    mask = ROOMS[room]()
    mm = I.material_map(torch.from_numpy(mask), "random", 7).numpy()
    o, g = pair(orc, mask, 32, [0.1] * 7, matmap=mm)
    check_classification(o, g)


@pytest.mark.parametrize("dims", [(45, 37, 19), (64, 20, 9), (33, 1, 70), (300, 7, 5)])
def test_mask_upload_bit_packed_and_byte_stream_agree(orc, dims, monkeypatch):
    """A host mask crosses PCIe bit-packed (host threads, AVX2) unless
    RAFD_MASK_BITS=0 streams its bytes: both give the oracle's classification,
    for any nonzero byte as "inside", x extents that are not multiples of 32,
    and a slab whose mask holds only its planes plus the two ghost planes."""
    nx, ny, nz = dims
    rng = np.random.default_rng(nx * 7 + ny)
    mask = rng.choice(np.array([0, 1, 7, 255], np.uint8), size=(nz, ny, nx), p=[0.15, 0.65, 0.1, 0.1])
    mm = I.material_map(torch.from_numpy((mask != 0).astype(np.uint8)), "random", 5).numpy()
    o = orc.OracleRoom((mask != 0).astype(np.uint8), LAM, 32, [0.1] * 5, matmap=mm)
    for bits in ("1", "0"):
        monkeypatch.setenv("RAFD_MASK_BITS", bits)
        g = rafd.Room(mask, LAM, 32, [0.1] * 5, matmap=mm)
        check_classification(o, g)
        g.destroy()
    # a slab's planes [z0, z1) from a mask that starts at plane z0 - 1
    z0, z1 = nz // 3, nz - nz // 3
    if z1 - z0 >= 1 and z0 >= 1:
        sub = np.ascontiguousarray(mask[z0 - 1:z1 + 1])
        msub = np.ascontiguousarray(mm[z0 - 1:z1 + 1])
        Ko = o.classification()[0]
        for bits in ("1", "0"):
            monkeypatch.setenv("RAFD_MASK_BITS", bits)
            g = rafd.Room(sub, LAM, 32, [0.1] * 5, matmap=msub, rank=0, nranks=3, z_begin=z0, z_end=z1,
                          mask_z0=z0 - 1, dims=(nx, ny, nz))
            Kg = g.get_classification()[0]
            assert np.array_equal(Kg, Ko[z0:z1]), bits
            g.destroy()


def test_classification_region_rule_and_device_inputs(orc):
    mask_t = I.dome_mask(64, 48, 40)
    mm_t = I.material_map(mask_t, "region", 8)
    o = orc.OracleRoom(mask_t.numpy(), LAM, 32, [0.1] * 8, matmap=mm_t.numpy())
    g = rafd.Room(mask_t.cuda(), LAM, 32, [0.1] * 8, matmap=mm_t.cuda())    # device pointers
    check_classification(o, g)


def test_c1_worked_example_bitwise(orc):
    """C1: 64^3 rigid box, fp64, 500 steps, impulse, 8 receivers."""
    cfg = I.CONFIGS["C1"]
    nx, ny, nz = cfg["dims"]
    mask = I.box_mask(nx, ny, nz).numpy()
    o, g = pair(orc, mask, 64, [0.0])
    src = I.source_position(cfg["dims"])
    rcv = I.receiver_positions(cfg["dims"])
    for r in (o, g):
        r.set_source(src, [1.0])
        r.set_receivers(rcv)
        r.step(cfg["steps"])
    ro, rg = o.read_receivers(), g.read_receivers()
    assert ro.shape == rg.shape == (8, 500)
    assert_close(ro, rg, 64, "receivers")
    assert_close(o.read_field()[0], g.read_field()[0], 64, "u^n")
    assert abs(g.energy() - 1.0) < 1e-12


@pytest.mark.parametrize("shape", ["lshape", "dome"])
def test_fi_mm_fp32_1000_steps(orc, shape):
    """C2-like (scaled down): FI-MM, M=4 region rule, fp32, 1000 steps."""
    mask = I.make_mask(shape, 48, 44, 40)
    mm = I.material_map(mask, "region", 4).numpy()
    mask = mask.numpy()
    beta0 = I.fi_beta_from_alpha(I.C2_ALPHAS)
    o, g = pair(orc, mask, 32, beta0, matmap=mm)
    src = I.source_position((48, 44, 40), mask)
    rcv = I.receiver_positions((48, 44, 40), mask)
    sig = I.gaussian_pulse(64, 6.0)
    for r in (o, g):
        r.set_source(src, sig)
        r.set_receivers(rcv)
        r.step(1000)
    assert_close(o.read_receivers(), g.read_receivers(), 32, "receivers")
    co, po = o.read_field()
    cg, pg = g.read_field()
    assert_close(co, cg, 32, "u^n")
    assert_close(po, pg, 32, "u^{n-1}")


@pytest.mark.parametrize("precision", [32, 64])
@pytest.mark.parametrize("MB", [1, 2, 3, 8])
def test_fd_mm_random_state(orc, precision, MB):
    """FD-MM with MB branches, 5 random materials, random initial fields and
    branch state, a source, 300 steps: fields and branch state bitwise."""
    mask = I.blob_mask(31, 27, 21, seed=MB, fill=0.8).numpy()
    mm = I.material_map(torch.from_numpy(mask), "random", 5).numpy()
    beta0, D, E, F = I.fd_tables(5, MB, seed=100 + MB)
    beta0 = np.array([0.0, 0.02, 0.0, 0.1, 0.3])
    o, g = pair(orc, mask, precision, beta0, D, E, F, matmap=mm)
    dt = np.float32 if precision == 32 else np.float64
    rng = np.random.default_rng(MB)
    up = rng.uniform(-1, 1, mask.shape).astype(dt)
    uc = rng.uniform(-1, 1, mask.shape).astype(dt)
    nb = o.nb
    v0 = rng.uniform(-0.1, 0.1, (MB, nb)).astype(dt)
    g0 = rng.uniform(-0.1, 0.1, (MB, nb)).astype(dt)
    src = I.snap_inside(mask, (15, 13, 10))
    rcv = [I.snap_inside(mask, p) for p in [(3, 3, 3), (20, 20, 15), (30, 26, 20)]]
    for r in (o, g):
        r.set_state(up, uc, v0, g0)
        r.set_source(src, I.gaussian_pulse(50, 5.0))
        r.set_receivers(rcv)
        r.step(300)
    check_classification(o, g)
    co, po = o.read_field()
    cg, pg = g.read_field()
    assert_close(co, cg, precision, "u^n")
    assert_close(po, pg, precision, "u^{n-1}")
    vo, go = o.read_branch_state()
    vg, gg = g.read_branch_state()
    assert_close(vo, vg, precision, "v")
    assert_close(go, gg, precision, "g")
    assert_close(o.read_receivers(), g.read_receivers(), precision, "receivers")
    eo, eg = o.energy(), g.energy()
    assert abs(eo - eg) <= 1e-9 * abs(eo)


@pytest.mark.parametrize("precision,MB", [(32, 0), (32, 3), (64, 2)])
def test_source_on_boundary_node_and_split_set_state(orc, precision, MB):
    """The source on a wall voxel (a boundary node, 0 < K < 6): the node's
    two-slot u_b ring must follow the source injection; the state is set in
    two calls (u^{n-1} only, then u^n only), each refreshing one ring slot."""
    mask = I.lshape_mask(40, 34, 22).numpy()
    mm = I.material_map(torch.from_numpy(mask), "random", 4).numpy()
    if MB:
        beta0, D, E, F = I.fd_tables(4, MB, seed=7)
    else:
        beta0, D, E, F = np.array([0.05, 0.2, 0.6, 0.9]), None, None, None
    o, g = pair(orc, mask, precision, beta0, D, E, F, matmap=mm)
    K = o.classification()[0]
    walls = np.argwhere((K > 0) & (K < 6))
    z, y, x = walls[len(walls) // 3]
    dt = np.float32 if precision == 32 else np.float64
    rng = np.random.default_rng(11)
    up = rng.uniform(-1, 1, mask.shape).astype(dt)
    uc = rng.uniform(-1, 1, mask.shape).astype(dt)
    o.set_state(up, uc)
    g.set_state(u_prev=up)
    g.set_state(u_curr=uc)
    for r in (o, g):
        r.set_source((int(x), int(y), int(z)), I.gaussian_pulse(80, 6.0))
        r.set_receivers([(int(x), int(y), int(z))])
        r.step(150)
    assert_close(o.read_receivers(), g.read_receivers(), precision, "receiver at the source")
    co, po = o.read_field()
    cg, pg = g.read_field()
    assert_close(co, cg, precision, "u^n")
    assert_close(po, pg, precision, "u^{n-1}")


def test_graph_and_direct_launches_agree(orc):
    """CUDA-graph replay (steps in blocks of 16) and one-by-one launches with
    profiling give identical bits."""
    mask = I.dome_mask(40, 40, 40).numpy()
    beta0, D, E, F = I.fd_tables(2, 3)
    mm = I.material_map(torch.from_numpy(mask), "random", 2).numpy()
    a = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    b = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    for r in (a, b):
        r.set_source((20, 20, 10), [1.0])
    a.step(67)
    b.set_profiling(True)
    for _ in range(67):
        b.step(1)
    t = b.get_kernel_times()
    fused = a.get_info()["fused"]
    assert t["volume_launches"] == 67 and t["boundary_launches"] == (0 if fused else 67)
    assert np.array_equal(a.read_field()[0], b.read_field()[0])
    # two kernels per step: volume + boundary (source/receivers in its last
    # block), or the fused volume kernel + source/receivers
    assert a.launch_count() == b.launch_count() == 67 * 2
    assert t["other_launches"] == (67 if fused else 0)


def test_degenerate_rooms(orc):
    # single voxel: isolated -> outside; no boundary; stepping is a no-op
    g = rafd.Room(np.ones((1, 1, 1), np.uint8), LAM, 32, [0.0])
    info = g.get_info()
    assert info["n_inside"] == 0 and info["n_boundary"] == 0 and info["isolated"] == 1
    g.step(5)
    with pytest.raises(rafd.RafdError) as e:
        g.set_source((0, 0, 0), [1.0])
    assert e.value.code == rafd.RAFD_E_OUTSIDE
    # all-outside mask
    g = rafd.Room(np.zeros((3, 4, 5), np.uint8), LAM, 64, [0.0])
    g.step(3)
    assert g.get_info()["n_inside"] == 0
    # 2x2x2: every voxel is a K=3 boundary node
    mask = np.ones((2, 2, 2), np.uint8)
    o, g = pair(orc, mask, 64, [0.3])
    for r in (o, g):
        r.set_source((1, 1, 1), [1.0, 0.5])
        r.step(50)
    assert_close(o.read_field()[0], g.read_field()[0], 64, "2x2x2")


def test_errors(orc):
    mask = I.lshape_mask(10, 10, 4).numpy()
    g = rafd.Room(mask, LAM, 32, [0.0, 0.1], matmap=np.zeros_like(mask))
    with pytest.raises(rafd.RafdError) as e:
        g.set_source((9, 9, 1), [1.0])                  # outside the L
    assert e.value.code == rafd.RAFD_E_OUTSIDE
    with pytest.raises(rafd.RafdError) as e:
        g.set_receivers([(1, 1, 1), (10, 0, 0)])       # off the grid
    assert e.value.code == rafd.RAFD_E_OUTSIDE
    mm = np.zeros_like(mask)
    mm[0, 0, 0] = 5
    with pytest.raises(rafd.RafdError) as e:
        rafd.Room(mask, LAM, 32, [0.0, 0.1], matmap=mm)
    assert e.value.code == rafd.RAFD_E_MATERIAL
    g.set_receivers([(1, 1, 1)])
    g.step(10)
    with pytest.raises(rafd.RafdError) as e:
        g.read_receivers(cap=5)
    assert e.value.code == rafd.RAFD_E_INVAL
    assert g.read_receivers(cap=10).shape == (1, 10)


@pytest.mark.parametrize("cfg", [0, 1, 2, 3])
@pytest.mark.parametrize("precision", [32, 64])
def test_volume_tile_configs_bitwise(orc, cfg, precision, monkeypatch):
    """Every tile configuration of the TMA volume kernel (RAFD_VOL_CFG) and the
    one-thread-per-voxel v0 kernel give the oracle's bits; the room (150x75x40)
    spans several tiles in x and y with ragged tails."""
    monkeypatch.setenv("RAFD_VOL_CFG", str(cfg))
    mask = I.dome_mask(150, 75, 40).numpy()
    mm = I.material_map(torch.from_numpy(mask), "region", 8).numpy()
    beta0, D, E, F = I.fd_tables(8, 3)
    o, g = pair(orc, mask, precision, beta0, D, E, F, matmap=mm)
    src = I.snap_inside(mask, (70, 30, 20))
    for r in (o, g):
        r.set_source(src, I.gaussian_pulse(30, 4.0))
        r.step(60)
    assert_close(o.read_field()[0], g.read_field()[0], precision, f"cfg {cfg}")
    if cfg == 0:
        monkeypatch.setenv("RAFD_VOLUME_KERNEL", "v0")
        g0 = rafd.Room(mask, LAM, precision, beta0, D, E, F, matmap=mm)
        g0.set_source(src, I.gaussian_pulse(30, 4.0))
        g0.step(60)
        assert_close(o.read_field()[0], g0.read_field()[0], precision, "v0")


@pytest.mark.parametrize("scheme", [1, 2])
@pytest.mark.parametrize("precision", [32, 64])
@pytest.mark.parametrize("kernel", ["tma", "v0"])
def test_single_kernel_schemes_bitwise(orc, scheme, precision, kernel, monkeypatch):
    """Listing 1 (one admittance) and Listing 6 (naive FI,
    constants loss1/loss2) as single kernels, vs the oracle's schemes."""
    if kernel == "v0":
        monkeypatch.setenv("RAFD_VOLUME_KERNEL", "v0")
    mask = I.dome_mask(150, 70, 40).numpy()
    beta = [0.27]
    c = 0.12
    kw = dict(scheme=scheme, loss1=1.0 / (1.0 + c), loss2=1.0 - c)
    o = orc.OracleRoom(mask, LAM, precision, beta)
    o.set_scheme(scheme, kw["loss1"], kw["loss2"])
    g = rafd.Room(mask, LAM, precision, beta, **kw)
    assert g.get_info()["scheme"] == scheme and g.get_info()["fused"] == 0
    src = I.snap_inside(mask, (70, 30, 20))
    rcv = [I.snap_inside(mask, p) for p in [(10, 30, 5), (75, 35, 20), (140, 40, 30)]]
    for r in (o, g):
        r.set_source(src, I.gaussian_pulse(30, 4.0))
        r.set_receivers(rcv)
        r.step(120)
    assert_close(o.read_field()[0], g.read_field()[0], precision, f"scheme {scheme}")
    assert_close(o.read_receivers(), g.read_receivers(), precision, "receivers")
    assert g.launch_count() == 2 * 120          # one volume kernel + source/receivers per step


def test_scheme_validation():
    mask = np.ones((6, 6, 6), np.uint8)
    with pytest.raises(rafd.RafdError) as e:
        rafd.Room(mask, LAM, 32, [0.1, 0.2], scheme=1)
    assert e.value.code == rafd.RAFD_E_INVAL
    with pytest.raises(rafd.RafdError) as e:
        rafd.Room(mask, LAM, 32, [0.0], D=[[1.0]], E=[[1.0]], F=[[1.0]], scheme=2)
    assert e.value.code == rafd.RAFD_E_INVAL


@pytest.mark.parametrize("shape", ["lshape", "dome"])
def test_empty_tile_skipping_bitwise(orc, shape, monkeypatch):
    """Tile-planes without inside voxels are skipped by the volume kernel
    (loads, compute, store); results equal the unskipped kernel and the oracle."""
    mask_t = I.make_mask(shape, 300, 260, 48)
    mm = I.material_map(mask_t, "region", 8).numpy()
    mask = mask_t.numpy()
    beta0, D, E, F = I.fd_tables(8, 3)
    src = I.source_position((300, 260, 48), mask)
    out = []
    for skip in ("1", "0"):
        monkeypatch.setenv("RAFD_SKIP_EMPTY", skip)
        g = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
        g.set_source(src, I.gaussian_pulse(40, 4.0))
        g.step(90)
        out.append(g.read_field()[0])
    o = orc.OracleRoom(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    o.set_source(src, I.gaussian_pulse(40, 4.0))
    o.step(90)
    assert_close(o.read_field()[0], out[0], 32, "skip")
    assert np.array_equal(out[0], out[1])


@pytest.mark.parametrize("precision,MB", [(32, 3), (64, 0)])
def test_checkpoint_resume_bitwise(precision, MB):
    """Save (u^n, u^{n-1}, v, g, n) after 70 steps, restore into a fresh room,
    continue 50 steps: bitwise equal to 120 uninterrupted steps (the source
    signal continues at the restored step index)."""
    mask = I.dome_mask(60, 50, 40).numpy()
    mm = I.material_map(torch.from_numpy(mask), "region", 8).numpy()
    if MB:
        beta0, D, E, F = I.fd_tables(8, MB)
    else:
        beta0, D, E, F = I.fi_beta_from_alpha(np.linspace(0.1, 0.8, 8)), None, None, None
    src = I.source_position((60, 50, 40), mask)
    sig = I.gaussian_pulse(200, 8.0)
    rcv = I.receiver_positions((60, 50, 40), mask)
    a = rafd.Room(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    a.set_source(src, sig)
    a.set_receivers(rcv)
    a.step(70)
    cur, prv = a.read_field()
    v, g = a.read_branch_state() if MB else (None, None)
    n = a.get_info()["steps"]
    a.step(50)
    b = rafd.Room(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    b.set_source(src, sig)
    b.set_receivers(rcv)
    b.set_state(prv, cur, v, g)
    b.set_step(n)
    b.step(50)
    assert np.array_equal(a.read_field()[0], b.read_field()[0])
    assert np.array_equal(a.read_receivers()[:, 70:], b.read_receivers())
