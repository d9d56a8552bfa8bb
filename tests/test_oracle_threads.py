"""The oracle's OpenMP loops (volume over z planes, boundary over nodes) give
results independent of the thread count, bit for bit (oracle/orc.c header).
No GPU."""
import math
import os

import numpy as np
import pytest

from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I

LAM = 1.0 / math.sqrt(3.0)


def _run(orc, threads, precision, fd, scheme=0):
    orc.set_threads(threads)
    mask_t = I.dome_mask(33, 29, 27)
    mask = mask_t.numpy()
    if fd:
        beta0, D, E, F = I.fd_tables(8, 3)
        beta0 = beta0 + 0.01
        mm = I.material_map(mask_t, "region", 8).numpy()
    else:
        beta0, D, E, F = ([0.05] if scheme else [0.01, 0.05, 0.2, 0.5]), None, None, None
        mm = None if scheme else I.material_map(mask_t, "random", 4).numpy()
    r = orc.OracleRoom(mask, LAM, precision, beta0, D, E, F, matmap=mm)
    if scheme:
        r.set_scheme(scheme, 0.9, 0.8)
    dt = np.float32 if precision == 32 else np.float64
    rng = np.random.default_rng(7)
    r.set_state((rng.uniform(-1, 1, mask.shape) * mask).astype(dt), (rng.uniform(-1, 1, mask.shape) * mask).astype(dt))
    r.set_source(I.source_position((33, 29, 27), mask), I.gaussian_pulse(20, 3.0))
    r.set_receivers(I.receiver_positions((33, 29, 27), mask))
    r.step(37)
    cur, prv = r.read_field()
    v, g = r.read_branch_state() if fd else (None, None)
    return cur, prv, v, g, r.read_receivers()


@pytest.mark.parametrize("precision,fd,scheme", [(32, True, 0), (64, True, 0), (32, False, 0), (64, False, 0),
                                                 (32, False, 1), (32, False, 2)])
def test_thread_count_does_not_change_results(orc, precision, fd, scheme):
    n = max(2, min(8, os.cpu_count() or 2))
    try:
        a = _run(orc, 1, precision, fd, scheme)
        b = _run(orc, n, precision, fd, scheme)
        c = _run(orc, 3, precision, fd, scheme)
    finally:
        orc.set_threads(os.cpu_count() or 1)
    for x, y, z in zip(a, b, c):
        if x is None:
            continue
        assert np.array_equal(x, y) and np.array_equal(x, z)
