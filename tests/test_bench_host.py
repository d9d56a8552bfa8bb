"""Host-side logic of bench.py (no GPU)."""
import numpy as np
import pytest

import bench
from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from paper_conf_ipps_stoltzfushsld21_b200 import rafd


@pytest.mark.parametrize("dims,p", [((20, 16, 40), 2), ((20, 16, 41), 3), ((12, 10, 64), 8), ((9, 7, 16), 4)])
def test_box_plan_matches_library_plan(dims, p):
    nx, ny, nz = dims
    lib_plan = rafd.rafd_slab_plan(I.box_mask(nx, ny, nz).numpy(), 32, 3, p)
    assert bench.slab_plan_box(nx, ny, nz, 32, 3, p) == lib_plan


def test_reference_arm_json_line(monkeypatch):
    class A:
        steps, warmup, config = 2, 1, "C1"
    out = bench.run_reference(A)
    assert out["impl"] == "reference" and out["value"] > 0
    assert out["cpu_baseline"]["kind"] == "oracle"
    assert out["e2e"]["h2d_bytes_per_step"] == 0
