"""Write tests/golden/c1_receivers.json from the closed form only.

    python tools/gen_c1_golden.py [--check]

Config C1 (pin P11): a 64^3 rigid box (every wall K < 6,
beta = 0), fp64, lambda = 1/sqrt(3), an impulse A = 1 added at (19, 25, 32) at
step 0, receivers at the eight fixed fractions of the dims, rec[j][n] =
u^{n+1}[rcv_j] for n = 0..499.

The rigid box's discrete Laplacian (masked 7-point, PAPER.md:349-357 with
K = number of inside neighbours) is diagonalised by the DCT-II basis
phi_m(i) = prod_d cos(pi m_d (i_d + 1/2) / N_d); mode m evolves as the
three-term recurrence a^{n+1} = 2 c_m a^n - a^{n-1}, c_m = 1 - 2 lambda^2
sum_d sin^2(pi m_d / (2 N_d)).  An impulse A at step 0 (u^0 = u^{-1} = 0,
u^1 = A delta_src) therefore gives a_m^{n+1} = A phi_m(src) / ||phi_m||^2
U_n(c_m), U_n the Chebyshev polynomial of the second kind, and
rec[j][n] = sum_m a_m^{n+1} phi_m(rcv_j).

This script evaluates U_n by its own recurrence (U_0 = 1, U_1 = 2c,
U_{n+1} = 2c U_n - U_{n-1}); the test (tests/test_oracle_pins.py,
c1_modal_receivers) evaluates the same closed form as sin((n+1) theta) /
sin(theta) -- two independent evaluations.  Nothing here calls the oracle or
the CUDA library.

The discrete energy (R11) after the impulse is H^{1/2} = A^2 = 1
(u^1 - u^0 = A delta, u^0 = 0 kills the edge term), conserved in a rigid room.
"""
from __future__ import annotations

import json
import math
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "tests", "golden", "c1_receivers.json")

DIMS = (64, 64, 64)
LAM = 1.0 / math.sqrt(3.0)
SRC = (19, 25, 32)  # floor((0.3, 0.4, 0.5) * 64)
FRACS = [(0.2, 0.2, 0.2), (0.2, 0.2, 0.6), (0.7, 0.3, 0.3), (0.3, 0.7, 0.3),
         (0.7, 0.3, 0.6), (0.3, 0.7, 0.6), (0.45, 0.45, 0.4), (0.25, 0.5, 0.45)]
STEPS = 500
PICKS = [(0, 99), (0, 249), (0, 499), (6, 99), (6, 249), (6, 499)]


def receivers():
    return [tuple(int(math.floor(f * d)) for f, d in zip(fr, DIMS)) for fr in FRACS]


def modal_traces(lam=LAM, dims=DIMS, src=SRC, rcvs=None, steps=STEPS, amp=1.0):
    rcvs = receivers() if rcvs is None else rcvs
    nx, ny, nz = dims
    ax = []
    # everything in x87 extended precision (64-bit mantissa): the recurrence's
    # rounding error grows ~n eps per mode, and c_m must carry more digits than
    # fp64 for U_499(c_m) to be exact to ~1e-16
    pi = np.longdouble("3.14159265358979323846264338327950288")
    for N in dims:
        m = np.arange(N, dtype=np.longdouble)[:, None]
        i = np.arange(N, dtype=np.longdouble)[None, :]
        ax.append((np.cos(pi * m * (i + np.longdouble(0.5)) / N),          # phi_m(i) along one axis
                   np.where(np.arange(N) == 0, np.longdouble(N), np.longdouble(N) / 2),  # ||phi_m||^2
                   np.sin(pi * m[:, 0] / (2 * N)) ** 2))
    (bx, nx2, sx), (by, ny2, sy), (bz, nz2, sz) = ax
    lam = np.longdouble(lam)  # the fp64 Courant number of the run, exactly
    c = 1 - 2 * lam * lam * (sz[:, None, None] + sy[None, :, None] + sx[None, None, :])
    w_src = (bz[:, src[2]][:, None, None] * by[:, src[1]][None, :, None] * bx[:, src[0]][None, None, :]) / \
        (nz2[:, None, None] * ny2[None, :, None] * nx2[None, None, :])
    out = np.zeros((len(rcvs), steps))
    weights = [amp * w_src * (bz[:, z][:, None, None] * by[:, y][None, :, None] * bx[:, x][None, None, :])
               for (x, y, z) in rcvs]
    u_prev = np.zeros_like(c)   # U_{-1} = 0
    u_cur = np.ones_like(c)     # U_0 = 1
    for n in range(steps):
        for j, w in enumerate(weights):
            out[j, n] = float((w * u_cur).sum())
        u_prev, u_cur = u_cur, 2 * c * u_cur - u_prev
    return out


def golden():
    rec = modal_traces()
    rcvs = receivers()
    return {
        "source": "SURVEY.md §8(c) pin P11 / §8(d) config C1: 64^3 rigid box, fp64, lambda = 1/sqrt(3), "
                  "impulse A=1 at (x,y,z)=(19,25,32) added at step 0, rec[j][n] = u^{n+1}[rcv_j]. Written by "
                  "tools/gen_c1_golden.py from the closed-form DCT-II modal synthesis rec[j][n] = sum_m A "
                  "phi_m(src) phi_m(rcv_j)/||phi_m||^2 U_n(cos theta_m), cos(theta_m) = 1 - 2 lambda^2 sum_d "
                  "sin^2(pi m_d / 2N) (U_n by the Chebyshev recurrence). Independent of the oracle; the test "
                  "also recomputes the modal sum itself (as sin((n+1) theta)/sin(theta)).",
        "lambda": LAM,
        "dims_xyz": list(DIMS),
        "source_xyz": list(SRC),
        "receivers_xyz": [list(r) for r in rcvs],
        "steps": STEPS,
        "values": [{"receiver": j, "n": n, "value": float(rec[j, n])} for j, n in PICKS],
        "sum_of_squares": float((rec ** 2).sum()),
        "peak_abs": float(np.abs(rec).max()),
        "energy": 1.0,
    }


def main():
    g = golden()
    if "--check" in sys.argv:
        old = json.load(open(OUT))
        for a, b in zip(old["values"], g["values"]):
            assert (a["receiver"], a["n"]) == (b["receiver"], b["n"])
            assert abs(a["value"] - b["value"]) < 1e-13, (a, b)
        assert abs(old["sum_of_squares"] - g["sum_of_squares"]) < 1e-12
        assert abs(old["peak_abs"] - g["peak_abs"]) < 1e-5
        print("c1_receivers.json agrees with the closed form")
        return
    with open(OUT, "w") as f:
        json.dump(g, f, indent=1)
        f.write("\n")
    print(f"wrote {OUT}")


if __name__ == "__main__":
    main()
