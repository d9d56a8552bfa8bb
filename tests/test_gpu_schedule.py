"""Unit scheduling of the two volume kernels: dynamic (atomic
unit counter, self-resetting) or static round-robin must give the same bits.
Small rooms default to static and large ones to dynamic (and skip the K plane
of uniform tile-planes only when large), so each test forces
one mode in a fresh process (the choice is read once per process) and checks
the single-step and two-step paths against the oracle, over several launches
(the counter must reset between them) and a slab group."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import math, sys
import numpy as np
sys.path.insert(0, %r)
from oracle import orc
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I, rafd
LAM = 1 / math.sqrt(3)
dims = (150, 90, 70)
mask = I.dome_mask(*dims).numpy()
mm = I.material_map(I.torch.from_numpy(mask), "region", 8).numpy()
b0, D, E, F = I.fd_tables(8, 3)
src = I.source_position(dims, mask)
rcv = I.receiver_positions(dims, mask)
sig = I.gaussian_pulse(30, 3.0)
o = orc.OracleRoom(mask, LAM, 32, b0, D, E, F, matmap=mm)
rooms = {}
for tb in (1, 2):
    r = rafd.Room(mask, LAM, 32, b0, D, E, F, matmap=mm)
    r.set_temporal_blocking(tb)
    rooms[tb] = r
plan = rafd.rafd_slab_plan(mask, 32, 3, 3)
slabs = [rafd.Room(mask, LAM, 32, b0, D, E, F, matmap=mm, rank=k, nranks=3, z_begin=a, z_end=b)
         for k, (a, b) in enumerate(plan)]
for s in slabs:
    s.set_temporal_blocking(2)
for r in list(rooms.values()) + slabs + [o]:
    r.set_source(src, sig)
    r.set_receivers(rcv)
for n in (7, 16, 9):  # direct launches, a CUDA graph of 16, an odd tail
    o.step(n)
    for r in rooms.values():
        r.step(n)
    rafd.rafd_step_group(slabs, n)
    ref = o.read_field()[0]
    for tb, r in rooms.items():
        assert np.array_equal(r.read_field()[0], ref), ("room", tb, n)
    assert np.array_equal(np.concatenate([s.read_field()[0] for s in slabs]), ref), ("slabs", n)
print("ok")
"""


@pytest.mark.parametrize("mode", ["0", "1"])
def test_dynamic_and_static_scheduling_bitwise(mode):
    # RAFD_K6: the K-plane skip of uniform tile-planes (default only in rooms of
    # >= 2^28 voxels) is exercised on this small room too
    env = dict(os.environ, RAFD_VOL_DYNAMIC=mode, RAFD_TB_DYNAMIC=mode, RAFD_K6=mode, RAFD_FUSED="0")
    # short z-chunks so that the dynamic counter hands out many units per launch
    env["RAFD_ZCHUNK_MAX"] = "8"
    env["RAFD_TB_ZCHUNK_MAX"] = "8"
    res = subprocess.run([sys.executable, "-c", SCRIPT % ROOT], env=env, capture_output=True, text=True,
                         timeout=600)
    assert res.returncode == 0 and "ok" in res.stdout, res.stdout[-2000:] + res.stderr[-4000:]
