"""Seeded random rooms vs the oracle (property: bitwise equality for any
geometry, materials, branch count, precision, scheme and tiling): dims from 1
to ~200 in x / ~140 in y / ~24 in z (ragged tiles, thin rooms, single rows),
Bernoulli / ellipsoid / L / dome shapes, random material maps, MB in 0..8,
fp32/fp64, random source and receivers, random initial state."""
import math

import numpy as np
import pytest
import torch

from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from paper_conf_ipps_stoltzfushsld21_b200 import rafd

pytestmark = pytest.mark.gpu


def case(seed):
    rng = np.random.default_rng(1000 + seed)
    nx = int(rng.integers(1, 200))
    ny = int(rng.integers(1, 140))
    nz = int(rng.integers(1, 24))
    shape = ["blob", "box", "ellipsoid", "lshape", "dome"][seed % 5]
    mask = I.make_mask(shape, nx, ny, nz, seed=seed)
    if shape == "blob":
        mask = I.blob_mask(nx, ny, nz, seed=seed, fill=float(rng.uniform(0.55, 0.95)))
    M = int(rng.integers(1, 9))
    mm = I.material_map(mask, "random", M).numpy()
    MB = int(rng.integers(0, 9)) if seed % 3 else 0
    prec = 32 if seed % 2 else 64
    lam = float(rng.uniform(0.3, 1 / math.sqrt(3)))
    if MB:
        beta0, D, E, F = I.fd_tables(M, MB, seed=seed)
        beta0 = rng.uniform(0, 0.2, M)
    else:
        beta0, D, E, F = rng.uniform(0, 1.0, M), None, None, None
    return mask.numpy(), mm, lam, prec, beta0, D, E, F, rng


@pytest.mark.parametrize("seed", list(range(24)))
def test_random_room_bitwise(orc, seed, monkeypatch):
    mask, mm, lam, prec, beta0, D, E, F, rng = case(seed)
    monkeypatch.setenv("RAFD_VOL_CFG", str(seed % 4))
    monkeypatch.setenv("RAFD_FUSED", "1" if seed % 4 == 3 else "0")
    o = orc.OracleRoom(mask, lam, prec, beta0, D, E, F, matmap=mm)
    g = rafd.Room(mask, lam, prec, beta0, D, E, F, matmap=mm)
    assert np.array_equal(o.classification()[0], g.get_classification()[0])
    inside = np.argwhere(o.classification()[0] > 0)
    if len(inside) == 0:
        g.step(3)
        return
    dt = np.float32 if prec == 32 else np.float64
    up = rng.uniform(-1, 1, mask.shape).astype(dt)
    uc = rng.uniform(-1, 1, mask.shape).astype(dt)
    pick = lambda: tuple(int(v) for v in inside[rng.integers(len(inside))][::-1])
    src = pick()
    rcv = [pick() for _ in range(int(rng.integers(1, 6)))]
    for r in (o, g):
        r.set_state(up, uc)
    sig = rng.uniform(-1, 1, 7)
    nsteps = int(rng.integers(1, 60))
    for r in (o, g):
        r.set_source(src, sig)
        r.set_receivers(rcv)
        r.step(nsteps)
    assert np.array_equal(o.read_field()[0], g.read_field()[0]), (seed, mask.shape)
    assert np.array_equal(o.read_receivers(), g.read_receivers())
    if D is not None:
        vo, go = o.read_branch_state()
        vg, gg = g.read_branch_state()
        assert np.array_equal(vo, vg) and np.array_equal(go, gg)


@pytest.mark.parametrize("seed", list(range(24)))
def test_random_room_two_step_bitwise(orc, seed, monkeypatch):
    """The same 24 rooms with temporal blocking (two steps per sweep, the shell
    recompute after the boundary update): bitwise equal to the oracle's single
    steps for any step count (odd counts end with one single step)."""
    mask, mm, lam, prec, beta0, D, E, F, rng = case(seed)
    monkeypatch.setenv("RAFD_FUSED", "0")
    o = orc.OracleRoom(mask, lam, prec, beta0, D, E, F, matmap=mm)
    g = rafd.Room(mask, lam, prec, beta0, D, E, F, matmap=mm)
    g.set_temporal_blocking(2)
    inside = np.argwhere(o.classification()[0] > 0)
    if len(inside) == 0:
        g.step(3)
        return
    dt = np.float32 if prec == 32 else np.float64
    up = rng.uniform(-1, 1, mask.shape).astype(dt)
    uc = rng.uniform(-1, 1, mask.shape).astype(dt)
    pick = lambda: tuple(int(v) for v in inside[rng.integers(len(inside))][::-1])
    src = pick()
    rcv = [pick() for _ in range(int(rng.integers(1, 6)))]
    sig = rng.uniform(-1, 1, 7)
    nsteps = int(rng.integers(1, 60))
    for r in (o, g):
        r.set_state(up, uc)
        r.set_source(src, sig)
        r.set_receivers(rcv)
        r.step(nsteps)
    assert np.array_equal(o.read_field()[0], g.read_field()[0]), (seed, mask.shape)
    assert np.array_equal(o.read_field()[1], g.read_field()[1])
    assert np.array_equal(o.read_receivers(), g.read_receivers())
    if D is not None:
        vo, go = o.read_branch_state()
        vg, gg = g.read_branch_state()
        assert np.array_equal(vo, vg) and np.array_equal(go, gg)
