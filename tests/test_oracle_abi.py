"""The oracle behind the product's C-ABI names (oracle/librafd_oracle.so,
SURVEY.md §8(b): "exports the same names and semantics (CPU, device/NCCL
fields ignored), implemented independently").  The product's own ctypes
binding (rafd.py) is pointed at that library, so these runs go through exactly
the calls a user of librafd.so makes -- on the CPU, no GPU needed."""
import contextlib
import math

import numpy as np
import pytest

from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from paper_conf_ipps_stoltzfushsld21_b200 import rafd

LAM = 1.0 / math.sqrt(3.0)


@contextlib.contextmanager
def oracle_abi(orc):
    """rafd.py bound to librafd_oracle.so for the duration."""
    orc.build()
    saved = (rafd.LIB_PATH, rafd._lib)
    rafd.LIB_PATH, rafd._lib = orc.ABI_LIB_PATH, None
    try:
        yield rafd.lib()
    finally:
        rafd.LIB_PATH, rafd._lib = saved


def test_exports_every_abi_name(orc):
    with oracle_abi(orc) as L:
        for name in rafd.ABI_SYMBOLS:
            assert hasattr(L, name), name
        assert L.rafd_version() == 1


def _case():
    mask_t = I.dome_mask(29, 23, 19)
    mask = mask_t.numpy()
    mm = I.material_map(mask_t, "region", 8).numpy()
    beta0, D, E, F = I.fd_tables(8, 3)
    rng = np.random.default_rng(5)
    up = (rng.uniform(-1, 1, mask.shape) * mask).astype(np.float32)
    uc = (rng.uniform(-1, 1, mask.shape) * mask).astype(np.float32)
    return mask, mm, beta0 + 0.01, D, E, F, up, uc


def test_room_through_the_abi_equals_the_oracle(orc):
    mask, mm, beta0, D, E, F, up, uc = _case()
    src = I.source_position((29, 23, 19), mask)
    rcv = I.receiver_positions((29, 23, 19), mask)
    sig = I.gaussian_pulse(12, 3.0)
    o = orc.OracleRoom(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    o.set_state(up, uc)
    o.set_source(src, sig)
    o.set_receivers(rcv)
    o.step(23)
    with oracle_abi(orc):
        r = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
        info = r.get_info()
        assert info["n_boundary"] == o.nb and info["z_end"] == 19
        assert info["bytes_per_step"] == info["volume_bytes"] + info["boundary_bytes"]
        assert info["boundary_bytes"] == o.nb * (6 + 12 + 48)
        r.set_temporal_blocking(2)  # accepted; the oracle steps one at a time
        r.set_state(up, uc)
        r.set_source(src, sig)
        r.set_receivers(rcv)
        r.step(10)
        # checkpoint, a new room resumed from it, 13 more steps
        cur, prv = r.read_field()
        v, g = r.read_branch_state()
        rec_a = r.read_receivers()
        r2 = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
        r2.set_state(prv, cur, v, g)
        r2.set_step(10)
        r2.set_source(src, sig)
        r2.set_receivers(rcv)
        r2.step(13)
        cur2, prv2 = r2.read_field()
        v2, g2 = r2.read_branch_state()
        rec = np.concatenate([rec_a, r2.read_receivers()], axis=1)
        cls = r2.get_classification()
        h = r2.energy()
        r.destroy()
        r2.destroy()
    co, po = o.read_field()
    vo, go = o.read_branch_state()
    assert np.array_equal(cur2, co) and np.array_equal(prv2, po)
    assert np.array_equal(v2, vo) and np.array_equal(g2, go)
    assert np.array_equal(rec, o.read_receivers())
    assert all(np.array_equal(a, b) for a, b in zip(cls, o.classification()))
    assert h == o.energy()


def test_errors_through_the_abi(orc):
    mask, mm, beta0, D, E, F, up, uc = _case()
    with oracle_abi(orc):
        with pytest.raises(rafd.RafdError) as e:
            rafd.Room(mask, 0.7, 32, beta0, D, E, F, matmap=mm)
        assert e.value.code == rafd.RAFD_E_UNSTABLE
        with pytest.raises(rafd.RafdError) as e:
            rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=np.full_like(mm, 9))
        assert e.value.code == rafd.RAFD_E_MATERIAL
        r = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
        with pytest.raises(rafd.RafdError) as e:
            r.set_source((0, 0, 0), [1.0])  # a corner of the dome's box is outside
        assert e.value.code == rafd.RAFD_E_OUTSIDE
        with pytest.raises(rafd.RafdError) as e:
            rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm, rank=0, nranks=2, z_begin=0, z_end=9)
        assert e.value.code == rafd.RAFD_E_STATE
        r.destroy()


@pytest.mark.parametrize("dims,p", [((21, 17, 40), 3), ((9, 8, 33), 5)])
def test_slab_plans_agree(orc, dims, p):
    """The oracle's and the product's slab plans (two implementations of
    SURVEY §8(e)'s cost-prefix split) agree."""
    mask = I.dome_mask(*dims).numpy()
    want = rafd.rafd_slab_plan(mask, 32, 3, p)
    with oracle_abi(orc):
        got = rafd.rafd_slab_plan(mask, 32, 3, p)
    assert got == want
