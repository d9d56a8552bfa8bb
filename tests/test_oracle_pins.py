"""Pins of the CPU oracle against what the paper and the mathematics fix
(SURVEY.md §8(c) P1-P11).  No GPU.

Each test is chosen so that a plausible mistake in the oracle (a dropped term,
a wrong sign or index, a transposed operand, a wrong neighbour count, a wrong
coefficient derivation) fails at least one of them.
"""
import json
import math
import os

import numpy as np
import pytest

from paper_conf_ipps_stoltzfushsld21_b200 import inputs as I
from tests.plain_fvtd import PlainFVTD

LAM = 1.0 / math.sqrt(3.0)
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def dct_mode(dims_xyz, m_xyz):
    """DCT-II basis function phi_m(i) = prod_d cos(pi m_d (i_d + 1/2) / N_d), [nz,ny,nx]."""
    p = [np.cos(np.pi * m * (np.arange(N) + 0.5) / N) for m, N in zip(m_xyz, dims_xyz)]
    return p[2][:, None, None] * p[1][None, :, None] * p[0][None, None, :]


def mode_theta(dims_xyz, m_xyz, lam):
    s = sum(math.sin(math.pi * m / (2 * N)) ** 2 for m, N in zip(m_xyz, dims_xyz))
    return 2.0 * math.asin(lam * math.sqrt(s))


# ---------------------------------------------------------------- P1 classification


def test_table2_box_boundary_counts(orc):
    """PAPER.md:1046-1052 (Table II): box boundary-point counts, exactly."""
    g = json.load(open(os.path.join(GOLDEN, "table2_box_counts.json")))
    for row in g["rows"]:
        nx, ny, nz = row["dims_xyz"]
        r = orc.OracleRoom(np.ones((nz, ny, nx), np.uint8), LAM, 32, [0.0])
        info = r.info()
        assert info["n_boundary"] == row["box_boundary_points"], row
        assert info["n_inside"] == nx * ny * nz
        del r


@pytest.mark.parametrize("dims", [(64, 64, 64), (13, 7, 5), (3, 4, 2)])
def test_box_k_histogram_closed_form(orc, dims):
    """K histogram of an nx*ny*nz box: corners K=3, edges K=4, faces K=5, rest 6."""
    nx, ny, nz = dims
    r = orc.OracleRoom(np.ones((nz, ny, nx), np.uint8), LAM, 64, [0.0])
    h = r.info()["k_hist"]
    a, b, c = nx - 2, ny - 2, nz - 2
    assert h[3] == 8
    assert h[4] == 4 * (a + b + c)
    assert h[5] == 2 * (a * b + a * c + b * c)
    assert h[6] == a * b * c
    assert h[0] == h[1] == h[2] == 0
    if dims == (64, 64, 64):
        assert (h[3], h[4], h[5], h[6]) == (8, 744, 23064, 238328)


def test_classification_brute_force(orc):
    """K, the ordered boundary list, K_b and mat_b on an irregular room vs a
    direct count of inside face neighbours per voxel (isolated voxels outside)."""
    mask = I.blob_mask(9, 8, 7, seed=3, fill=0.6).numpy()
    mask[0, 0, 0] = 1                     # carve one isolated inside voxel
    mask[0, 0, 1] = mask[0, 1, 0] = mask[1, 0, 0] = 0
    matmap = I.material_map(I.torch.from_numpy(mask), "random", 5).numpy()
    r = orc.OracleRoom(mask, LAM, 32, [0.1] * 5, matmap=matmap)
    K, bidx, Kb, matb = r.classification()
    nz, ny, nx = mask.shape
    Kref = np.zeros_like(K)
    for z in range(nz):
        for y in range(ny):
            for x in range(nx):
                if not mask[z, y, x]:
                    continue
                cnt = 0
                for dz, dy, dx in ((1, 0, 0), (-1, 0, 0), (0, 1, 0), (0, -1, 0), (0, 0, 1), (0, 0, -1)):
                    zz, yy, xx = z + dz, y + dy, x + dx
                    if 0 <= zz < nz and 0 <= yy < ny and 0 <= xx < nx and mask[zz, yy, xx]:
                        cnt += 1
                Kref[z, y, x] = cnt
    assert np.array_equal(K, Kref)
    flat = Kref.reshape(-1)
    want = np.flatnonzero((flat > 0) & (flat < 6))
    assert np.array_equal(bidx, want)
    assert np.all(np.diff(bidx) > 0)
    assert np.array_equal(Kb, flat[want])
    assert np.array_equal(matb, matmap.reshape(-1)[want])
    info = r.info()
    assert info["isolated"] == int(((mask.reshape(-1) > 0) & (flat == 0)).sum())
    assert info["isolated"] > 0  # the fixture does exercise the isolated-voxel rule


# ---------------------------------------------------------------- P2/P3 closed-form modes


@pytest.mark.parametrize("precision,tol", [(64, 1e-11), (32, 2e-3)])
def test_rigid_box_dct_modes(orc, precision, tol):
    """Rigid cuboid: the DCT-II basis is an exact discrete mode,
    u^n = cos(n w) phi with cos w = 1 - 2 l^2 sum_d sin^2(pi m_d / 2N_d)."""
    dims = (12, 10, 8)
    nx, ny, nz = dims
    dt = np.float64 if precision == 64 else np.float32
    for m in [(1, 0, 0), (2, 1, 3), (11, 9, 7), (5, 0, 6)]:
        phi = dct_mode(dims, m)
        w = mode_theta(dims, m, LAM)
        r = orc.OracleRoom(np.ones((nz, ny, nx), np.uint8), LAM, precision, [0.0])
        r.set_state(u_prev=(math.cos(w) * phi).astype(dt), u_curr=phi.astype(dt))
        nsteps = 1000
        r.step(nsteps)
        cur, _ = r.read_field()
        err = np.abs(cur - math.cos(nsteps * w) * phi).max()
        assert err < tol, (m, err)


def test_rigid_box_modal_frequencies(orc):
    """Cuboid-room modal frequencies: the spectrum of an impulse response in a
    rigid 12x10x8 box peaks at the discrete modal frequencies theta_m, which
    approach the continuous f_m = (c/2) sqrt(sum (m_d/(N_d h))^2) as h -> 0."""
    dims = (12, 10, 8)
    nx, ny, nz = dims
    r = orc.OracleRoom(np.ones((nz, ny, nx), np.uint8), LAM, 64, [0.0])
    r.set_source((1, 2, 3), [1.0, -1.0])      # zero-mean: no DC drift
    r.set_receivers([(9, 8, 6)])
    nfft = 8192
    r.step(nfft)
    rec = r.read_receivers()[0]
    spec = np.abs(np.fft.rfft(rec * np.hanning(nfft)))
    omega = 2 * np.pi * np.arange(spec.size) / nfft
    for m in [(1, 0, 0), (0, 1, 0), (1, 1, 0), (0, 0, 1), (2, 0, 0)]:
        th = mode_theta(dims, m, LAM)
        k = int(round(th / (2 * np.pi) * nfft))
        lo, hi = k - 3, k + 4
        kpk = lo + int(np.argmax(spec[lo:hi]))
        assert abs(omega[kpk] - th) <= 2 * np.pi / nfft, (m, omega[kpk], th)
        # the peak is a true local maximum (a mode, not leakage)
        assert spec[kpk] > spec[kpk - 3] and spec[kpk] > spec[kpk + 3]
    # continuous limit of the discrete frequency (closed form only)
    for N in (10, 100, 1000):
        th = mode_theta((N, N, N), (2, 1, 3), LAM)
        cont = math.pi * LAM * math.sqrt((2 / N) ** 2 + (1 / N) ** 2 + (3 / N) ** 2)
        assert abs(th / cont - 1) < 3.0 / N ** 2 * 10


# ---------------------------------------------------------------- P11 worked example C1


def c1_modal_receivers(lam, dims, src, rcvs, nsteps, amp=1.0):
    """Independent closed-form receiver traces of an impulse in a rigid box:
    rec[j][n] = sum_m A phi_m(src) phi_m(rcv_j)/||phi_m||^2 sin((n+1) th_m)/sin th_m."""
    nx, ny, nz = dims
    axes = []
    for N, s in zip(dims, range(3)):
        mm = np.arange(N)
        i = np.arange(N)
        basis = np.cos(np.pi * mm[:, None] * (i[None, :] + 0.5) / N)   # [m, i]
        norm = np.where(mm == 0, N, N / 2.0)
        sin2 = np.sin(np.pi * mm / (2 * N)) ** 2
        axes.append((basis, norm, sin2))
    (bx, nxn, sx), (by, nyn, sy), (bz, nzn, sz) = axes
    # mode grid flattened as [mz, my, mx]
    S = (sz[:, None, None] + sy[None, :, None] + sx[None, None, :]).reshape(-1)
    cos_th = 1 - 2 * lam * lam * S
    th = np.arccos(np.clip(cos_th, -1, 1))
    norm = (nzn[:, None, None] * nyn[None, :, None] * nxn[None, None, :]).reshape(-1)
    phi_src = (bz[:, src[2]][:, None, None] * by[:, src[1]][None, :, None] * bx[:, src[0]][None, None, :]).reshape(-1)
    W = []
    for (x, y, z) in rcvs:
        phi_r = (bz[:, z][:, None, None] * by[:, y][None, :, None] * bx[:, x][None, None, :]).reshape(-1)
        W.append(amp * phi_src * phi_r / norm)
    W = np.array(W)                                    # [R, modes]
    n1 = np.arange(1, nsteps + 1, dtype=np.float64)
    out = np.zeros((len(rcvs), nsteps))
    chunk = 8192
    for c0 in range(0, th.size, chunk):
        t = th[c0:c0 + chunk]
        st = np.sin(t)
        dc = st < 1e-300
        U = np.where(dc[:, None], n1[None, :], np.sin(np.outer(t, n1)) / np.where(dc, 1.0, st)[:, None])
        out += W[:, c0:c0 + chunk] @ U
    return out


def test_c1_worked_example(orc):
    """C1: whole pipeline incl. source/receiver semantics vs
    the closed-form modal synthesis, and the stored closed-form values."""
    g = json.load(open(os.path.join(GOLDEN, "c1_receivers.json")))
    nx, ny, nz = g["dims_xyz"]
    r = orc.OracleRoom(np.ones((nz, ny, nx), np.uint8), g["lambda"], 64, [0.0])
    r.set_source(g["source_xyz"], [1.0])
    r.set_receivers(g["receivers_xyz"])
    r.step(g["steps"])
    rec = r.read_receivers()
    assert rec.shape == (8, g["steps"])
    ref = c1_modal_receivers(g["lambda"], (nx, ny, nz), g["source_xyz"], g["receivers_xyz"], g["steps"])
    assert np.abs(rec - ref).max() < 1e-12
    for v in g["values"]:
        assert abs(rec[v["receiver"], v["n"]] - v["value"]) < 1e-13
    assert abs((rec ** 2).sum() - g["sum_of_squares"]) < 1e-12
    assert abs(np.abs(rec).max() - g["peak_abs"]) < 1e-5
    assert abs(r.energy() - g["energy"]) < 1e-12


# ---------------------------------------------------------------- P4 discrete energy


def _rand_state(mask, seed, dt):
    rng = np.random.default_rng(seed)
    up = rng.uniform(-1, 1, mask.shape).astype(dt)
    uc = rng.uniform(-1, 1, mask.shape).astype(dt)
    return up * mask, uc * mask


def _energy_series(r, n):
    hs = []
    for _ in range(n):
        r.step(1)
        hs.append(r.energy())
    return np.array(hs)


ROOMS = {
    "ellipsoid": lambda: I.ellipsoid_mask(14, 12, 10).numpy(),
    "blob": lambda: I.blob_mask(10, 9, 8, seed=11, fill=0.85).numpy(),
    "lshape": lambda: I.lshape_mask(10, 8, 6).numpy(),
}


@pytest.mark.parametrize("room", list(ROOMS))
def test_energy_conserved_rigid_and_lossless(orc, room):
    """H^{n+1/2} is conserved to rounding with rigid walls (FI beta=0) and with
    lossless FD branches (E=F=0, beta0=0)."""
    mask = ROOMS[room]()
    up, uc = _rand_state(mask, 5, np.float64)
    r = orc.OracleRoom(mask, LAM, 64, [0.0])
    r.set_state(up, uc)
    h = _energy_series(r, 300)
    assert h.min() > 0
    assert np.abs(h / h[0] - 1).max() < 1e-12
    beta0, D, E, F = I.fd_tables(3, 3, lossless=True)
    mm = I.material_map(I.torch.from_numpy(mask), "random", 3).numpy()
    r = orc.OracleRoom(mask, LAM, 64, beta0, D, E, F, matmap=mm)
    r.set_state(up, uc)
    h = _energy_series(r, 300)
    assert np.abs(h / h[0] - 1).max() < 1e-12
    # fp32: conserved to single-precision rounding
    up32, uc32 = _rand_state(mask, 5, np.float32)
    r = orc.OracleRoom(mask, LAM, 32, [0.0])
    r.set_state(up32, uc32)
    h = _energy_series(r, 300)
    assert np.abs(h / h[0] - 1).max() < 2e-5


@pytest.mark.parametrize("room", list(ROOMS))
def test_energy_decays_lossy(orc, room):
    """Passive FI (beta > 0) and passive FD walls: H non-increasing every step,
    and strictly decreasing overall."""
    mask = ROOMS[room]()
    up, uc = _rand_state(mask, 9, np.float64)
    mm = I.material_map(I.torch.from_numpy(mask), "random", 4).numpy()
    r = orc.OracleRoom(mask, LAM, 64, [0.01, 0.1, 0.5, 2.0], matmap=mm)
    r.set_state(up, uc)
    h = _energy_series(r, 300)
    assert np.all(np.diff(h) <= 1e-13 * h[0])
    assert h[-1] < 0.9 * h[0]
    beta0, D, E, F = I.fd_tables(4, 3)
    beta0 = np.array([0.0, 0.05, 0.0, 0.2])
    r = orc.OracleRoom(mask, LAM, 64, beta0, D, E, F, matmap=mm)
    r.set_state(up, uc)
    h = _energy_series(r, 300)
    assert np.all(np.diff(h) <= 1e-13 * h[0])
    assert h[-1] < 0.99 * h[0]


def _balance_rhs(mask, K, bidx, lam, beta0, D, E, F, matb, u_prev, u_next, v0, v1, g0, g1):
    """Right-hand side of the exact one-step energy balance (SURVEY.md Appendix
    A.1, reading R11), from the fields and branch states alone:
      H^{n+1/2} - H^{n-1/2} = - sum_{boundary i} lam (6-K_i) [ beta0 du^2 / 2
                              + sum_b ( 2 E_b mu_v_b^2 + F_b (g'_b - g_b)^2 ) ]
    with du = u^{n+1} - u^{n-1} at the node and mu_v_b = (v'_b + v_b) / 2.
    It follows from multiplying the FVTD update by du and the
    branch ODE 2D(v'-v) + E(v'+v) + 2F g' = du (Listing 4 with R5's BI, DI;
    PAPER.md:426-440) by mu_v."""
    flat_prev, flat_next = u_prev.reshape(-1), u_next.reshape(-1)
    a = lam * (6.0 - K.reshape(-1)[bidx].astype(np.float64))
    du = flat_next[bidx].astype(np.float64) - flat_prev[bidx].astype(np.float64)
    diss = np.asarray(beta0, np.float64)[matb] * du * du / 2.0
    for b in range(v0.shape[0]):
        mu = (v1[b].astype(np.float64) + v0[b].astype(np.float64)) / 2.0
        dg = g1[b].astype(np.float64) - g0[b].astype(np.float64)
        diss = diss + 2.0 * E[matb, b] * mu * mu + F[matb, b] * dg * dg
    return -(a * diss).sum()


@pytest.mark.parametrize("room", list(ROOMS))
def test_energy_balance_exact(orc, room):
    """Exact per-step energy balance (not just its sign): every term of the
    oracle's H -- kinetic, edge, and the boundary D v^2 and F g^2 terms -- is
    pinned by the dissipation computed independently from the states.  FD
    tables with D, E, F > 0 and beta0 > 0, random field and branch state; an
    FI room with beta0 > 0; an R-free (E = 0) table so that the F terms carry
    the whole dissipation of the branches."""
    mask = ROOMS[room]()
    mm = I.material_map(I.torch.from_numpy(mask), "random", 4).numpy()
    rng = np.random.default_rng(2024)
    beta0, D, E, F = I.fd_tables(4, 3)
    beta0 = np.array([0.0, 0.05, 0.3, 0.02])
    E_free = E.copy()
    E_free[:, :] = 0.0
    cases = [("fi", beta0 + 0.01, None, None, None),
             ("fd", beta0, D, E, F),
             ("fd_E0", beta0 * 0, D, E_free, F)]
    for name, b0, Dc, Ec, Fc in cases:
        r = orc.OracleRoom(mask, LAM, 64, b0, Dc, Ec, Fc, matmap=mm)
        K, bidx_c, Kb, matb = r.classification()
        nz, ny, nx = mask.shape
        z, rem = np.divmod(bidx_c, ny * nx)
        y, x = np.divmod(rem, nx)
        bflat = (z * ny + y) * nx + x
        up, uc = _rand_state(mask, 31, np.float64)
        nb, MB = r.nb, (0 if Dc is None else Dc.shape[1])
        v = rng.uniform(-1, 1, (MB, nb))
        g = rng.uniform(-1, 1, (MB, nb))
        r.set_state(up, uc, v if MB else None, g if MB else None)
        for _ in range(5):
            h0 = r.energy()
            u_n, u_prev = r.read_field()
            v0, g0 = r.read_branch_state() if MB else (np.zeros((0, nb)), np.zeros((0, nb)))
            r.step(1)
            h1 = r.energy()
            u_next, _ = r.read_field()
            v1, g1 = r.read_branch_state() if MB else (np.zeros((0, nb)), np.zeros((0, nb)))
            rhs = _balance_rhs(mask, K, bflat, LAM, b0, Dc if MB else None,
                               Ec if MB else None, Fc if MB else None, matb,
                               u_prev, u_next, v0, v1, g0, g1)
            assert rhs < 0, name
            assert abs((h1 - h0) - rhs) <= 1e-12 * abs(h0), (name, h1 - h0, rhs)
            if MB:
                # the F g^2 part of H alone is O(1) here: a dropped or scaled
                # term would break the balance by that much
                a = LAM * (6.0 - Kb.astype(np.float64))
                fg = (a * (Fc[matb, :].T * g1 * g1).sum(0)).sum()
                assert fg > 1e-3 * abs(h1), name


# ---------------------------------------------------------------- P5 stability limit


def test_lambda_validation(orc):
    mask = np.ones((4, 4, 4), np.uint8)
    orc.OracleRoom(mask, LAM, 32, [0.0])                         # 1/sqrt(3) accepted
    for bad in (LAM * 1.0001, 0.0, -0.5, float("nan")):
        with pytest.raises(orc.OracleError) as e:
            orc.OracleRoom(mask, bad, 32, [0.0])
        assert e.value.code == -2


def test_box_stability_threshold(orc):
    """The exact box threshold l* = 1/sqrt(sum_d cos^2(pi/2N_d)) (spectral radius
    of the masked Laplacian): just below it the field stays bounded, just above
    it grows exponentially (raw path: no l check)."""
    dims = (16, 14, 12)
    nx, ny, nz = dims
    lstar = 1.0 / math.sqrt(sum(math.cos(math.pi / (2 * N)) ** 2 for N in dims))
    assert lstar > LAM
    mask = np.ones((nz, ny, nx), np.uint8)
    up, uc = _rand_state(mask, 1, np.float64)
    res = {}
    for f in (0.999, 1.02):
        r = orc.OracleRoom(mask, lstar * f, 64, [0.0], raw={"beta": [0.0]})
        r.set_state(up, uc)
        r.step(600)
        cur, _ = r.read_field()
        res[f] = np.abs(cur).max()
    assert res[0.999] < 50.0
    assert res[1.02] > 1e6


# ---------------------------------------------------------------- P6 spectral radius


def _step_matrix(orc, mask, lam, matmap, **kw):
    """Dense one-step map on the state [u^{n-1}, u^n, v, g] built column by column."""
    r = orc.OracleRoom(mask, lam, 64, matmap=matmap, **kw)
    K, _, _, _ = r.classification()
    inside = np.flatnonzero(K.reshape(-1) > 0)
    nb, MB = r.nb, r.MB
    n_in = inside.size
    dim = 2 * n_in + 2 * MB * nb
    A = np.zeros((dim, dim))
    for c in range(dim):
        e = np.zeros(dim)
        e[c] = 1.0
        up = np.zeros(mask.size); uc = np.zeros(mask.size)
        up[inside] = e[:n_in]; uc[inside] = e[n_in:2 * n_in]
        v = e[2 * n_in:2 * n_in + MB * nb].reshape(MB, nb)
        g = e[2 * n_in + MB * nb:].reshape(MB, nb)
        r.set_state(up.reshape(mask.shape), uc.reshape(mask.shape), v, g)
        r.step(1)
        cur, prv = r.read_field()
        v2, g2 = r.read_branch_state()
        A[:, c] = np.concatenate([prv.reshape(-1)[inside], cur.reshape(-1)[inside],
                                  v2.reshape(-1), g2.reshape(-1)])
    return A


def test_spectral_radius_passive_vs_inconsistent(orc):
    """Passive FD tables: rho(one-step map) = 1.  Listing-4 tables with
    beta = 0.5 * sum_b BI (inconsistent with reading R5): rho > 1 (unstable)."""
    mask = np.ones((3, 3, 4), np.uint8)
    mask[0, 0, 0] = 0
    mm = I.material_map(I.torch.from_numpy(mask), "random", 2).numpy()
    beta0, D, E, F = I.fd_tables(2, 2)
    A = _step_matrix(orc, mask, LAM, mm, beta0=beta0, D=D, E=E, F=F)
    rho = np.abs(np.linalg.eigvals(A)).max()
    assert abs(rho - 1.0) < 1e-6
    BI = 1.0 / (2 * D + E + F)
    DI = 2 * D - E - F
    bad = {"beta": 0.5 * BI.sum(axis=1), "BI": BI, "D": D, "DI": DI, "F": F}
    A = _step_matrix(orc, mask, LAM, mm, beta0=beta0, raw=bad)
    rho_bad = np.abs(np.linalg.eigvals(A)).max()
    assert rho_bad > 1.001          # unstable: an eigenvalue outside the unit circle


# ---------------------------------------------------------------- P7 reductions


@pytest.mark.parametrize("precision", [32, 64])
def test_fd_single_resistive_branch_equals_fi(orc, precision):
    """An FD table with beta0 = 0 and one branch D = F = 0, E = 1/beta reduces
    Listing 4 to Listing 3 with admittance beta: bitwise equal fields.
    Zero-padded branches (D = E = F = 0) are no-ops."""
    dt = np.float32 if precision == 32 else np.float64
    mask = I.blob_mask(11, 9, 8, seed=2, fill=0.85).numpy()
    mm = I.material_map(I.torch.from_numpy(mask), "random", 3).numpy()
    betas = np.array([0.25, 0.5, 0.125])          # 1/(1/beta) == beta exactly
    up, uc = _rand_state(mask, 4, dt)
    fi = orc.OracleRoom(mask, LAM, precision, betas, matmap=mm)
    D = np.zeros((3, 1)); F = np.zeros((3, 1)); E = (1.0 / betas)[:, None]
    fd = orc.OracleRoom(mask, LAM, precision, np.zeros(3), D, E, F, matmap=mm)
    D3 = np.zeros((3, 3)); E3 = np.zeros((3, 3)); F3 = np.zeros((3, 3)); E3[:, 1] = 1.0 / betas
    fd3 = orc.OracleRoom(mask, LAM, precision, np.zeros(3), D3, E3, F3, matmap=mm)
    src = I.snap_inside(mask, (5, 4, 4))
    for r in (fi, fd, fd3):
        r.set_state(up, uc)
        r.set_source(src, I.gaussian_pulse(40, 5.0))
        r.step(150)
    a = fi.read_field()[0]
    b = fd.read_field()[0]
    c = fd3.read_field()[0]
    assert np.array_equal(a, b)
    assert np.array_equal(a, c)
    assert np.abs(a).max() > 1e-3


# ---------------------------------------------------------------- P8 outside invariance


def test_outside_stays_positive_zero(orc):
    mask = I.blob_mask(10, 9, 8, seed=7, fill=0.7).numpy()
    beta0, D, E, F = I.fd_tables(2, 3)
    mm = I.material_map(I.torch.from_numpy(mask), "random", 2).numpy()
    r = orc.OracleRoom(mask, LAM, 32, beta0, D, E, F, matmap=mm)
    up, uc = _rand_state(np.ones_like(mask), 3, np.float32)   # nonzero everywhere: set_state must clear outside
    r.set_state(up, uc)
    r.set_source(I.snap_inside(mask, (5, 5, 4)), [1.0])
    r.step(100)
    K, _, _, _ = r.classification()
    cur, prv = r.read_field()
    out = K == 0
    assert out.sum() > 0
    for f in (cur, prv):
        assert np.all(f[out] == 0) and not np.any(np.signbit(f[out]))


# ---------------------------------------------------------------- P9 plain definition


def _fd_case(seed, M, MB):
    rng = np.random.default_rng(seed)
    D = rng.uniform(0, 2, (M, MB)); E = rng.uniform(0, 2, (M, MB)); F = rng.uniform(0, 2, (M, MB))
    beta0 = rng.uniform(0, 0.5, M)
    return beta0, D, E, F


@pytest.mark.parametrize("kind", ["FI", "FD"])
def test_plain_definition_single_step(orc, kind):
    """One step of Listings 2-4 equals the per-node linear solve of the FVTD +
    branch equations (with random nonzero branch state), to rounding."""
    mask = I.blob_mask(8, 7, 6, seed=21, fill=0.8).numpy()
    mm = I.material_map(I.torch.from_numpy(mask), "random", 3).numpy()
    if kind == "FI":
        beta0, D, E, F = np.array([0.05, 0.3, 1.0]), None, None, None
    else:
        beta0, D, E, F = _fd_case(1, 3, 3)
    r = orc.OracleRoom(mask, LAM, 64, beta0, D, E, F, matmap=mm)
    p = PlainFVTD(mask, LAM, beta0, D, E, F, matmap=mm)
    up, uc = _rand_state(mask, 8, np.float64)
    rng = np.random.default_rng(99)
    MB = 0 if D is None else D.shape[1]
    v0 = rng.uniform(-1, 1, (MB, r.nb)); g0 = rng.uniform(-1, 1, (MB, r.nb))
    r.set_state(up, uc, v0 if MB else None, g0 if MB else None)
    p.set_fields(up, uc)
    assert np.array_equal(p.canonical()[p.bnd], r.classification()[1])
    p.v, p.g = v0.copy(), g0.copy()
    r.step(1)
    p.step()
    cur, prv = r.read_field()
    assert np.abs(cur - p.field(p.u)).max() < 1e-13
    assert np.array_equal(prv, uc * (r.classification()[0] > 0))
    if MB:
        v, g = r.read_branch_state()
        assert np.abs(v - p.v).max() < 1e-12
        assert np.abs(g - p.g).max() < 1e-12


@pytest.mark.parametrize("kind", ["FI", "FD"])
def test_plain_definition_iterated(orc, kind):
    """200 steps on an irregular 7x6x5 room: oracle vs the plain definition."""
    mask = I.blob_mask(7, 6, 5, seed=5, fill=0.8).numpy()
    mm = I.material_map(I.torch.from_numpy(mask), "random", 4).numpy()
    if kind == "FI":
        beta0, D, E, F = np.random.default_rng(4).uniform(0, 1, 4), None, None, None
    else:
        beta0, D, E, F = _fd_case(2, 4, 2)
    r = orc.OracleRoom(mask, LAM, 64, beta0, D, E, F, matmap=mm)
    p = PlainFVTD(mask, LAM, beta0, D, E, F, matmap=mm)
    up, uc = _rand_state(mask, 6, np.float64)
    r.set_state(up, uc)
    p.set_fields(up, uc)
    for _ in range(200):
        p.step()
    r.step(200)
    cur, _ = r.read_field()
    ref = p.field(p.u)
    assert np.abs(cur - ref).max() < 1e-12 * max(1.0, np.abs(ref).max())


# ---------------------------------------------------------------- P10 duct reflection


def _reflection_exact(omega, lam, a, Y):
    xi = 2 * np.arcsin(np.sin(omega / 2) / lam)
    gamma = (a / lam) * Y * np.sin(omega)
    return (np.exp(-1j * xi) - 1 + 1j * gamma) / (1 - 1j * gamma - np.exp(1j * xi))


def _duct_run(orc, n, beta0, D, E, F, steps, x_src=3000, x_rcv=4000, sigma=4.0):
    mask = np.ones((1, 1, n), np.uint8)
    mm = np.zeros((1, 1, n), np.uint8)
    mm[0, 0, n - 1] = 1
    r = orc.OracleRoom(mask, LAM, 64, beta0, D, E, F, matmap=mm)
    x = np.arange(n)
    u0 = np.exp(-0.5 * ((x - x_src) / sigma) ** 2).reshape(1, 1, n)
    r.set_state(u0, u0)
    r.set_receivers([(x_rcv, 0, 0)])
    r.step(steps)
    return r.read_receivers()[0]


@pytest.mark.parametrize("kind", ["FI", "FD"])
def test_duct_reflection_coefficient(orc, kind):
    """Frequency-resolved pin of the boundary kernels: |R(w)| measured in a
    1-voxel duct (the last node carries the material, a = 6-K = 5 absorbing
    faces) vs the exact discrete reflection coefficient
    R = (e^{-i xi} - 1 + i gamma)/(1 - i gamma - e^{i xi}), sin(w/2) = l sin(xi/2),
    gamma = (a/l) Y(e^{iw}) sin w,
    Y(z) = beta0 + sum_b (1+z^-1)/[2D(1-z^-1) + E(1+z^-1) + F(1+z^-1)/(1-z^-1)]."""
    steps = 14000       # reflected window [6000, 14000): the FD ring-down has decayed to 1e-11
    if kind == "FI":
        beta0 = np.array([0.0, 0.04]); D = E = F = None
    else:
        rng = np.random.default_rng(17)
        D = np.zeros((2, 2)); E = np.zeros((2, 2)); F = np.zeros((2, 2))
        D[1] = rng.uniform(0.5, 3, 2); E[1] = rng.uniform(0.5, 3, 2); F[1] = rng.uniform(0.01, 0.2, 2)
        beta0 = np.array([0.0, 0.0])
    test = _duct_run(orc, 6000, beta0, D, E, F, steps)
    ref = _duct_run(orc, 20000, beta0, D, E, F, steps)
    nfft = 1 << 15
    inc = np.zeros(nfft); inc[:4000] = ref[:4000]
    refl = np.zeros(nfft); refl[:8000] = (test - ref)[6000:14000]
    Fi = np.fft.rfft(inc); Fr = np.fft.rfft(refl)
    omega = 2 * np.pi * np.arange(Fi.size) / nfft
    sel = (np.abs(Fi) > 1e-3 * np.abs(Fi).max()) & (omega > 0.005) & (omega < 0.6)
    assert sel.sum() > 500
    meas = np.abs(Fr[sel]) / np.abs(Fi[sel])
    z = np.exp(1j * omega[sel])
    if kind == "FI":
        Y = beta0[1] * np.ones_like(z)
    else:
        zi = 1 / z
        Y = beta0[1] + sum((1 + zi) / (2 * D[1, b] * (1 - zi) + E[1, b] * (1 + zi) + F[1, b] * (1 + zi) / (1 - zi))
                           for b in range(2))
    exact = np.abs(_reflection_exact(omega[sel], LAM, 5.0, Y))
    assert np.abs(meas - exact).max() < 1e-7
    assert exact.max() - exact.min() > (0.01 if kind == "FI" else 0.1)   # genuinely frequency-resolved


# ---------------------------------------------------------------- validation


def test_parameter_validation(orc):
    mask = np.ones((4, 5, 6), np.uint8)
    with pytest.raises(orc.OracleError) as e:
        orc.OracleRoom(mask, LAM, 32, [-0.1])
    assert e.value.code == -3
    with pytest.raises(orc.OracleError) as e:
        orc.OracleRoom(mask, LAM, 32, [0.0], D=[[-1.0]], E=[[1.0]], F=[[1.0]])
    assert e.value.code == -3
    with pytest.raises(orc.OracleError) as e:
        orc.OracleRoom(mask, LAM, 16, [0.0])
    assert e.value.code == -1
    mm = np.zeros_like(mask); mm[0, 0, 0] = 2
    with pytest.raises(orc.OracleError) as e:
        orc.OracleRoom(mask, LAM, 32, [0.0, 0.1], matmap=mm)
    assert e.value.code == -5
    mm[0, 0, 0] = 0; mm[2, 2, 2] = 7                          # interior voxel: never read
    orc.OracleRoom(mask, LAM, 32, [0.0, 0.1], matmap=mm)
    mask2 = mask.copy(); mask2[1, 1, 1] = 0
    r = orc.OracleRoom(mask2, LAM, 32, [0.0])
    with pytest.raises(orc.OracleError) as e:
        r.set_source((1, 1, 1), [1.0])
    assert e.value.code == -4
    with pytest.raises(orc.OracleError) as e:
        r.set_receivers([(0, 0, 0), (6, 0, 0)])
    assert e.value.code == -4


def test_fp32_is_single_precision_and_close_to_fp64(orc):
    """fp32 path really runs in single precision (differs from fp64) but stays
    within single-precision accumulation error of it."""
    mask = I.ellipsoid_mask(16, 14, 12).numpy()
    beta0, D, E, F = I.fd_tables(4, 3)
    mm = I.material_map(I.torch.from_numpy(mask), "random", 4).numpy()
    out = {}
    for p in (32, 64):
        r = orc.OracleRoom(mask, LAM, p, beta0, D, E, F, matmap=mm)
        r.set_source(I.snap_inside(mask, (8, 7, 6)), I.gaussian_pulse(60, 6.0))
        r.set_receivers([I.snap_inside(mask, (4, 4, 4))])
        r.step(400)
        out[p] = r.read_receivers()[0]
    d = np.abs(out[32] - out[64]).max() / np.abs(out[64]).max()
    assert 0 < d < 1e-2            # fp32 vs fp64 differ by 3e-4..7e-3 of peak


# ---------------------------------------------------------------- single-kernel schemes (f3)


def test_listing1_equals_two_kernel_fi(orc):
    """Listing 1 (one kernel) and Listings 2+3 (two kernels)
    are the same update written two ways: equal to rounding for beta > 0
    (1e-12 of peak after 300 fp64 steps), and bitwise for beta = 0 (the
    boundary branch degenerates to t - prev exactly)."""
    mask = I.blob_mask(12, 11, 9, seed=31, fill=0.85).numpy()
    up, uc = _rand_state(mask, 12, np.float64)
    for beta, bitwise in ((0.3, False), (0.0, True)):
        a = orc.OracleRoom(mask, LAM, 64, [beta])
        b = orc.OracleRoom(mask, LAM, 64, [beta])
        b.set_scheme(1)
        for r in (a, b):
            r.set_state(up, uc)
            r.step(300)
        fa, fb = a.read_field()[0], b.read_field()[0]
        if bitwise:
            assert np.array_equal(fa, fb)
        else:
            assert not np.array_equal(fa, fb)            # really a different rounding sequence
            assert np.abs(fa - fb).max() <= 1e-12 * np.abs(fa).max()
    with pytest.raises(orc.OracleError):
        orc.OracleRoom(mask, LAM, 64, [0.1, 0.2]).set_scheme(1)   # one admittance only


def test_listing1_energy_decays(orc):
    mask = I.ellipsoid_mask(14, 12, 10).numpy()
    up, uc = _rand_state(mask, 13, np.float64)
    r = orc.OracleRoom(mask, LAM, 64, [0.2])
    r.set_scheme(1)
    r.set_state(up, uc)
    h = _energy_series(r, 200)
    assert np.all(np.diff(h) <= 1e-13 * h[0]) and h[-1] < 0.9 * h[0]


def test_listing6_naive_rigid_is_dct_mode(orc):
    """Listing 6 with loss1 = loss2 = 1 is the rigid
    leapfrog summed in LIFT's neighbour order: the DCT-II modes are exact."""
    dims = (12, 10, 8)
    nx, ny, nz = dims
    for m in [(2, 1, 3), (11, 9, 7)]:
        phi = dct_mode(dims, m)
        w = mode_theta(dims, m, LAM)
        r = orc.OracleRoom(np.ones((nz, ny, nx), np.uint8), LAM, 64, [0.0])
        r.set_scheme(2, 1.0, 1.0)
        r.set_state(u_prev=math.cos(w) * phi, u_curr=phi)
        r.step(1000)
        assert np.abs(r.read_field()[0] - math.cos(1000 * w) * phi).max() < 1e-11


def test_listing6_naive_energy(orc):
    """With loss1 = 1/(1+c), loss2 = 1-c the naive update is
    u+ - 2u + u- = l^2 sum(u_j - u) - c (u+ - u-) at boundary points: H is
    non-increasing for c > 0 and conserved for c = 0."""
    mask = I.ellipsoid_mask(14, 12, 10).numpy()
    up, uc = _rand_state(mask, 14, np.float64)
    for c in (0.0, 0.15):
        r = orc.OracleRoom(mask, LAM, 64, [0.0])
        r.set_scheme(2, 1.0 / (1.0 + c), 1.0 - c)
        r.set_state(up, uc)
        h = _energy_series(r, 200)
        if c == 0.0:
            assert np.abs(h / h[0] - 1).max() < 1e-12
        else:
            assert np.all(np.diff(h) <= 1e-13 * h[0]) and h[-1] < 0.95 * h[0]
