"""Seeded synthetic inputs shared by the tests, bench.py and smoke().

This module holds NO arithmetic of the method (no classification, no stencil,
no boundary update, no coefficient derivation): it only draws the rooms,
material maps, physical material parameters, source signals and receiver
positions that both the CUDA path and the CPU oracle are fed (DESIGN.md
"Input recipe").  Masks are built with torch so the same code
can run on the CPU (oracle-sized rooms) or on the GPU (the 1.1e9-voxel hall,
which would take tens of seconds in numpy); integer ops only, so both give the
same bytes.

Shapes of the paper's workloads: box rooms (Table II),
"dome-shaped" rooms (geometry not given, reading
R12 in DESIGN.md), L-shaped rooms (north_star "non-cuboid (L-shaped/dome)").
"""
from __future__ import annotations

import math

import numpy as np
import torch

# ---------------------------------------------------------------- room masks


def _centres(n, device):
    return torch.arange(n, device=device, dtype=torch.float64) + 0.5


def box_mask(nx, ny, nz, device="cpu"):
    """Cuboid room: every voxel of the nx*ny*nz grid is inside."""
    return torch.ones((nz, ny, nx), dtype=torch.uint8, device=device)


def lshape_mask(nx, ny, nz, device="cpu"):
    """L-shaped room: outside iff x >= nx/2 and y >= ny/2 (all z)."""
    m = torch.ones((nz, ny, nx), dtype=torch.uint8, device=device)
    m[:, ny // 2:, nx // 2:] = 0
    return m


def dome_mask(nx, ny, nz, device="cpu"):
    """Dome: elliptic cylinder (semi-axes nx/2, ny/2) up to z = nz/2, capped by a
    half-ellipsoid of semi-axis nz/2 above; cell centres (i+1/2).  256^3 gives
    N_in = 10 979 828 and Nb = 228 556."""
    cx, cy, cz = _centres(nx, device), _centres(ny, device), _centres(nz, device)
    rx = ((cx - nx / 2) / (nx / 2)) ** 2
    ry = ((cy - ny / 2) / (ny / 2)) ** 2
    rz = ((cz - nz / 2) / (nz / 2)) ** 2
    rxy = ry[:, None] + rx[None, :]                     # [ny, nx]
    upper = (cz > nz / 2)[:, None, None]                # [nz,1,1]
    r = rxy[None, :, :] + torch.where(upper, rz[:, None, None], torch.zeros_like(rz)[:, None, None])
    return (r <= 1.0).to(torch.uint8)


def blob_mask(nx, ny, nz, seed, fill=0.8, device="cpu"):
    """Irregular room for small tests: each voxel inside with probability
    `fill` (seeded); produces isolated voxels, K=1..5 of every kind."""
    g = torch.Generator().manual_seed(int(seed))
    m = (torch.rand((nz, ny, nx), generator=g, dtype=torch.float64) < fill).to(torch.uint8)
    return m.to(device)


def ellipsoid_mask(nx, ny, nz, device="cpu"):
    """Inscribed ellipsoid (cell centres)."""
    cx, cy, cz = _centres(nx, device), _centres(ny, device), _centres(nz, device)
    r = (((cz - nz / 2) / (nz / 2)) ** 2)[:, None, None] + \
        (((cy - ny / 2) / (ny / 2)) ** 2)[None, :, None] + \
        (((cx - nx / 2) / (nx / 2)) ** 2)[None, None, :]
    return (r <= 1.0).to(torch.uint8)


SHAPES = {"box": box_mask, "lshape": lshape_mask, "dome": dome_mask, "ellipsoid": ellipsoid_mask}


def make_mask(shape, nx, ny, nz, device="cpu", seed=0):
    if shape == "blob":
        return blob_mask(nx, ny, nz, seed, device=device)
    return SHAPES[shape](nx, ny, nz, device=device)


# ---------------------------------------------------------------- materials


def _splitmix64(x: torch.Tensor) -> torch.Tensor:
    """splitmix64 on int64 tensors (wrapping arithmetic), used only to scatter
    material ids for the `random` rule."""
    def srl(v, k):  # logical shift right on int64
        return (v >> k) & ((1 << (64 - k)) - 1)
    c1 = -7046029254386353131   # 0x9E3779B97F4A7C15 as int64
    c2 = -4658895280553007687   # 0xBF58476D1CE4E5B9
    c3 = -7723592293110705685   # 0x94D049BB133111EB
    z = x + c1
    z = (z ^ srl(z, 30)) * c2
    z = (z ^ srl(z, 27)) * c3
    return z ^ srl(z, 31)


def material_map(mask: torch.Tensor, rule: str, M: int) -> torch.Tensor:
    """Per-voxel material ids (uint8 [nz,ny,nx]); only boundary voxels' values
    are ever read.  Rules (SURVEY.md §8(d) "Material assignment"):

    region, M=8: m = index of the first missing face neighbour in the order
        -z,+z,-y,+y,-x,+x (0..5); floor (m=0) with nx/4 <= x < 3nx/4 -> 6;
        walls (m in 2..5) with z >= 3nz/4 -> 7.
    region, M=4: -z -> 0, +z -> 1, +-y -> 2, +-x -> 3.
    random: splitmix64(0x5EED ^ canonical index) mod M.
    uniform: all 0.
    """
    nz, ny, nx = mask.shape
    dev = mask.device
    if rule == "uniform":
        return torch.zeros_like(mask)
    if rule == "random":
        idx = torch.arange(nz * ny * nx, device=dev, dtype=torch.int64)
        h = _splitmix64(idx ^ 0x5EED)
        return torch.remainder(h, M).to(torch.uint8).reshape(nz, ny, nx)
    if rule != "region":
        raise ValueError(rule)
    p = torch.nn.functional.pad(mask, (1, 1, 1, 1, 1, 1))
    missing = [
        p[:-2, 1:-1, 1:-1] == 0,  # -z
        p[2:, 1:-1, 1:-1] == 0,   # +z
        p[1:-1, :-2, 1:-1] == 0,  # -y
        p[1:-1, 2:, 1:-1] == 0,   # +y
        p[1:-1, 1:-1, :-2] == 0,  # -x
        p[1:-1, 1:-1, 2:] == 0,   # +x
    ]
    first = torch.full(mask.shape, 255, dtype=torch.uint8, device=dev)
    for k in range(5, -1, -1):            # later assignments win -> lowest k wins
        first = torch.where(missing[k], torch.tensor(k, dtype=torch.uint8, device=dev), first)
    del missing, p
    first = torch.where(first == 255, torch.zeros_like(first), first)
    if M == 4:
        lut = torch.tensor([0, 1, 2, 2, 3, 3], dtype=torch.uint8, device=dev)
        return lut[first.long()]
    if M != 8:
        raise ValueError("region rule needs M = 4 or 8")
    z = torch.arange(nz, device=dev)[:, None, None]
    x = torch.arange(nx, device=dev)[None, None, :]
    out = first.clone()
    floor_aud = (first == 0) & (x >= nx // 4) & (x < (3 * nx) // 4)
    out = torch.where(floor_aud, torch.tensor(6, dtype=torch.uint8, device=dev), out)
    upper = (first >= 2) & (first <= 5) & (z >= (3 * nz) // 4)
    out = torch.where(upper, torch.tensor(7, dtype=torch.uint8, device=dev), out)
    return out


def fi_beta_from_alpha(alpha):
    """Normal-incidence absorption alpha -> FI admittance
    beta = (1 - sqrt(1-alpha)) / (1 + sqrt(1-alpha))."""
    a = np.asarray(alpha, dtype=np.float64)
    r = np.sqrt(1.0 - a)
    return (1.0 - r) / (1.0 + r)


C2_ALPHAS = [0.05, 0.2, 0.5, 0.9]


def fd_tables(M, MB, seed=20210517, lossless=False):
    """Physical per-branch parameters of a passive series-RLC branch
    (SURVEY.md §8(d) "FD tables"): per (m, b) in row-major order draw
    theta0 ~ U[0.05, 0.8] rad/sample, Q ~ U[0.5, 5], b0 ~ U[0.01, 0.3];
    E = 1/b0, D = Q*E/theta0, F = D*theta0^2, beta0 = 0.
    lossless=True sets E = F = 0 (energy-conservation test tables)."""
    rng = np.random.default_rng(seed)
    D = np.zeros((M, MB)); E = np.zeros((M, MB)); F = np.zeros((M, MB))
    for m in range(M):
        for b in range(MB):
            th0 = rng.uniform(0.05, 0.8)
            Q = rng.uniform(0.5, 5.0)
            b0 = rng.uniform(0.01, 0.3)
            E[m, b] = 1.0 / b0
            D[m, b] = Q * E[m, b] / th0
            F[m, b] = D[m, b] * th0 * th0
    if lossless:
        E[:] = 0.0
        F[:] = 0.0
    return np.zeros(M), D, E, F


# ---------------------------------------------------------------- source / receivers

RECEIVER_FRACTIONS = [(0.2, 0.2, 0.2), (0.2, 0.2, 0.6), (0.7, 0.3, 0.3), (0.3, 0.7, 0.3),
                      (0.7, 0.3, 0.6), (0.3, 0.7, 0.6), (0.45, 0.45, 0.4), (0.25, 0.5, 0.45)]
SOURCE_FRACTION = (0.3, 0.4, 0.5)


def _frac_pos(f, dims):
    return tuple(int(math.floor(fi * d)) for fi, d in zip(f, dims))


def snap_inside(mask_np: np.ndarray, xyz):
    """Nearest voxel (Euclidean) whose mask is set; ties broken by lowest
    canonical index.  (Callers use rooms without isolated voxels.)"""
    nz, ny, nx = mask_np.shape
    x, y, z = xyz
    if mask_np[z, y, x]:
        return (x, y, z)
    zz, yy, xx = np.nonzero(mask_np)
    d2 = (xx - x) ** 2 + (yy - y) ** 2 + (zz - z) ** 2
    best = np.flatnonzero(d2 == d2.min())
    canon = (zz[best] * ny + yy[best]) * nx + xx[best]
    k = best[np.argmin(canon)]
    return (int(xx[k]), int(yy[k]), int(zz[k]))


def source_position(dims, mask_np=None):
    p = _frac_pos(SOURCE_FRACTION, dims)
    return snap_inside(mask_np, p) if mask_np is not None else p


def receiver_positions(dims, mask_np=None):
    ps = [_frac_pos(f, dims) for f in RECEIVER_FRACTIONS]
    return [snap_inside(mask_np, p) if mask_np is not None else p for p in ps]


def impulse(amplitude=1.0):
    return np.array([amplitude], dtype=np.float64)


def gaussian_pulse(n, width, seed=None):
    """Zero-mean differentiated Gaussian (no DC component), length n."""
    t = np.arange(n, dtype=np.float64)
    c = n / 2.0
    return -(t - c) / width * np.exp(-0.5 * ((t - c) / width) ** 2)


def random_field(shape, seed, dtype=np.float32, scale=1.0):
    """Seeded uniform field in [-scale, scale) (float32 values are generated in
    float32 so they are exactly representable for both sides)."""
    rng = np.random.default_rng(seed)
    return (rng.uniform(-scale, scale, size=shape)).astype(dtype)


# ---------------------------------------------------------------- the BASELINE.json configs

CONFIGS = {
    # name: (shape, (nx, ny, nz), MB, M, material rule, precision, steps)
    "C1": dict(shape="box", dims=(64, 64, 64), MB=0, M=1, rule="uniform", precision=64, steps=500,
               beta0=[0.0]),
    "C2a": dict(shape="lshape", dims=(256, 256, 256), MB=0, M=4, rule="region", precision=32,
                steps=2000),
    "C2b": dict(shape="dome", dims=(256, 256, 256), MB=0, M=4, rule="region", precision=32,
                steps=2000),
    "C3": dict(shape="box", dims=(512, 384, 256), MB=3, M=8, rule="region", precision=32,
               steps=1000),
    "C3d": dict(shape="box", dims=(512, 384, 256), MB=3, M=8, rule="region", precision=64,
                steps=1000),
    "C4": dict(shape="box", dims=(1536, 1024, 704), MB=3, M=8, rule="region", precision=32,
               steps=1000),
    "C5": dict(shape="box", dims=(2048, 1536, 2560), MB=3, M=8, rule="region", precision=32,
               steps=200),
}


def config_materials(cfg):
    """(beta0, D, E, F) for a config: FI configs get beta from C2_ALPHAS (M=4)
    or the explicit beta0; FD configs get fd_tables(M, MB)."""
    if cfg["MB"] == 0:
        if "beta0" in cfg:
            return np.asarray(cfg["beta0"], dtype=np.float64), None, None, None
        return fi_beta_from_alpha(C2_ALPHAS[: cfg["M"]]), None, None, None
    return fd_tables(cfg["M"], cfg["MB"])


def region_map_box(nx, ny, nz, z_lo, z_hi, M=8, device="cpu"):
    """The `region` material rule for a BOX room, generated directly for planes
    [z_lo, z_hi) only (slab-sized inputs for the large halls).  Equals
    material_map(box_mask(nx, ny, nz), "region", M)[z_lo:z_hi] (tested)."""
    z = torch.arange(z_lo, z_hi, device=device)[:, None, None]
    y = torch.arange(ny, device=device)[None, :, None]
    x = torch.arange(nx, device=device)[None, None, :]
    shape = (z_hi - z_lo, ny, nx)
    first = torch.full(shape, 255, dtype=torch.int16, device=device)
    faces = [z == 0, z == nz - 1, y == 0, y == ny - 1, x == 0, x == nx - 1]
    for k in range(5, -1, -1):
        first = torch.where(faces[k].expand(shape), torch.tensor(k, dtype=torch.int16, device=device), first)
    first = torch.where(first == 255, torch.zeros_like(first), first)
    if M == 4:
        lut = torch.tensor([0, 1, 2, 2, 3, 3], dtype=torch.uint8, device=device)
        return lut[first.long()]
    out = first.clone()
    out = torch.where((first == 0) & (x >= nx // 4) & (x < (3 * nx) // 4), torch.tensor(6, dtype=torch.int16, device=device), out)
    out = torch.where((first >= 2) & (first <= 5) & (z >= (3 * nz) // 4), torch.tensor(7, dtype=torch.int16, device=device), out)
    return out.to(torch.uint8)
