"""The library's device memory cache (include/rafd.h rafd_release_cached_memory):
rooms created in memory a destroyed room left dirty in the cache still match the
oracle bit for bit, and the cache can be handed back to the driver."""
import math

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu
LAM = 1.0 / math.sqrt(3.0)


def _room_pair(orc, rafd, I, seed, tb):
    mask_t = I.dome_mask(45, 37, 29)
    mask = mask_t.numpy()
    mm = I.material_map(mask_t, "region", 8).numpy()
    beta0, D, E, F = I.fd_tables(8, 3)
    rng = np.random.default_rng(seed)
    up = (rng.uniform(-1, 1, mask.shape) * mask).astype(np.float32)
    uc = (rng.uniform(-1, 1, mask.shape) * mask).astype(np.float32)
    g = rafd.Room(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    o = orc.OracleRoom(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    if tb == 2:
        g.set_temporal_blocking(2)
    src, rcv = I.source_position((45, 37, 29), mask), I.receiver_positions((45, 37, 29), mask)
    for r in (g, o):
        r.set_state(up, uc)
        r.set_source(src, I.gaussian_pulse(16, 3.0))
        r.set_receivers(rcv)
        r.step(33)
    return g, o


def test_rooms_in_reused_pool_memory_match_the_oracle(orc):
    from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
    from paper_conf_ipps_stoltzfushsld21_b200 import rafd
    for it in range(4):
        g, o = _room_pair(orc, rafd, I, seed=it, tb=1 + it % 2)
        assert np.array_equal(g.read_field()[0], o.read_field()[0])
        assert np.array_equal(g.read_receivers(), o.read_receivers())
        v, gg = g.read_branch_state()
        vo, go = o.read_branch_state()
        assert np.array_equal(v, vo) and np.array_equal(gg, go)
        g.destroy()  # its memory goes back to the cache, dirty
    free0 = torch.cuda.mem_get_info(0)[0]
    rafd.rafd_release_cached_memory(0)
    assert torch.cuda.mem_get_info(0)[0] >= free0
    with pytest.raises(rafd.RafdError):
        rafd.rafd_release_cached_memory(-1)
