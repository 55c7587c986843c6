"""Seeded, partition-independent synthetic inputs.

This module is shared by the oracle side (tests, bench's cpu_baseline leg)
and by the host side of the product path (host buffers for the e2e leg).
It holds NONE of the method's arithmetic (no stencil, map, reduce, CG or
LBM step): only the counter-based generator and the problem set-up values
(domain masks, the manufactured right-hand side).  The CUDA library has
its own independent implementation of the same counter-based generator
(``nb_field_fill``); ``tests/test_gpu_parity.py`` checks the two are
byte-identical.

Generator:

    gidx = x + Nx*(y + Ny*z) + c*Nx*Ny*Nz             (global, not per partition)
    mix64(z): z ^= z>>30; z *= 0xBF58476D1CE4E5B9; z ^= z>>27;
              z *= 0x94D049BB133111EB; z ^= z>>31      (all mod 2^64)
    h = mix64(seed*0x9E3779B97F4A7C15 + gidx + 1)
    real uniform:  u = (h>>11) * 2^-53;  v = lo + (hi-lo)*u   (fp64, no fma)
    int uniform in [lo, hi]:  v = lo + (h mod (hi-lo+1))
"""
from __future__ import annotations

import numpy as np

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
GOLDEN = np.uint64(0x9E3779B97F4A7C15)
MIX1 = np.uint64(0xBF58476D1CE4E5B9)
MIX2 = np.uint64(0x94D049BB133111EB)


def mix64(z: np.ndarray) -> np.ndarray:
    """SplitMix64 finaliser, elementwise on uint64 (wrapping arithmetic)."""
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z ^ (z >> np.uint64(30))
        z = z * MIX1
        z = z ^ (z >> np.uint64(27))
        z = z * MIX2
        z = z ^ (z >> np.uint64(31))
    return z


def hashes(seed: int, gidx: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        base = np.uint64(seed) * GOLDEN
        return mix64(base + np.asarray(gidx, dtype=np.uint64) + np.uint64(1))


def gidx_range(start: int, count: int) -> np.ndarray:
    return np.arange(start, start + count, dtype=np.uint64)


def uniform(dims, card: int = 1, seed: int = 1, lo: float = -1.0, hi: float = 1.0,
            dtype=np.float64, z_range=None) -> np.ndarray:
    """Real uniform field, dense logical view [c][z][y][x] (x fastest).

    ``z_range=(z0, z1)`` returns only those global planes (still indexed by
    global gidx), so a bounded sample of a huge field can be generated."""
    nx, ny, nz = dims
    z0, z1 = (0, nz) if z_range is None else z_range
    out = np.empty((card, z1 - z0, ny, nx), dtype=dtype)
    plane = nx * ny
    for c in range(card):
        start = c * plane * nz + z0 * plane
        h = hashes(seed, gidx_range(start, (z1 - z0) * plane))
        u = (h >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
        v = lo + (hi - lo) * u  # numpy: two separately rounded ops, no fma
        out[c] = v.reshape(z1 - z0, ny, nx).astype(dtype)
    return out if card > 1 else out[0]


def int_uniform(dims, card: int = 1, seed: int = 1, lo: int = -8, hi: int = 8,
                dtype=np.float64, z_range=None) -> np.ndarray:
    """Integer-valued field in [lo, hi] (exact in fp32/fp64)."""
    nx, ny, nz = dims
    z0, z1 = (0, nz) if z_range is None else z_range
    out = np.empty((card, z1 - z0, ny, nx), dtype=dtype)
    plane = nx * ny
    span = np.uint64(hi - lo + 1)
    for c in range(card):
        start = c * plane * nz + z0 * plane
        h = hashes(seed, gidx_range(start, (z1 - z0) * plane))
        v = (h % span).astype(np.int64) + lo
        out[c] = v.reshape(z1 - z0, ny, nx).astype(dtype)
    return out if card > 1 else out[0]


def poisson_poly_rhs(dims, dtype=np.float64, z_range=None) -> np.ndarray:
    """Right-hand side b = h^2 f of the manufactured Poisson problem
    (SURVEY.md §8(c) c5 pin 1): u*(x,y,z) = g(x)g(y)g(z), g(t) = t(1-t),
    x_i = (i+1) h, h = 1/(N+1) per axis, f = 2[g(y)g(z) + g(x)g(z) + g(x)g(y)].

    Operation order (mirrored by the CUDA fill, which uses _rn intrinsics):
      t = (i+1)*h ; g = t*(1-t) ; f = ((gy*gz + gx*gz) + gx*gy) * 2 ; b = (h*h)*f
    A cubic grid is assumed (one h); the product path checks the same.
    """
    nx, ny, nz = dims
    assert nx == ny == nz, "manufactured RHS is defined on a cube"
    h = 1.0 / (nx + 1)
    z0, z1 = (0, nz) if z_range is None else z_range
    t = np.arange(1, nx + 1, dtype=np.float64) * h
    g = t * (1.0 - t)
    gz = g[z0:z1][:, None, None]
    gy = g[None, :, None]
    gx = g[None, None, :]
    f = ((gy * gz + gx * gz) + gx * gy) * 2.0
    return ((h * h) * f).astype(dtype)


def poisson_poly_solution(n: int) -> np.ndarray:
    """u* on the N^3 grid (the exact discrete solution of A u = b above)."""
    h = 1.0 / (n + 1)
    t = np.arange(1, n + 1, dtype=np.float64) * h
    g = t * (1.0 - t)
    return g[:, None, None] * g[None, :, None] * g[None, None, :]


def sphere_mask(n: int, r_frac: float = 0.41528) -> np.ndarray:
    """Free-form sparse domain of config C4: cell
    (x,y,z) is active iff its centre lies in the sphere of radius r_frac*N
    centred in the box: (x+1/2-N/2)^2 + (y+1/2-N/2)^2 + (z+1/2-N/2)^2 <= r^2.
    Returns uint8 [z][y][x]."""
    r = r_frac * n
    c = np.arange(n, dtype=np.float64) + 0.5 - n / 2.0
    c2 = c * c
    out = np.empty((n, n, n), dtype=np.uint8)
    for z in range(n):
        out[z] = ((c2[:, None] + c2[None, :]) + c2[z] <= r * r)
    return out


def cube_mask(n: int, frac: float) -> np.ndarray:
    """Solid cube of edge round(frac^(1/3) * N) anchored at the origin
    (the Fig. 9 'sparsity ratio' read as the active volume fraction)."""
    e = max(1, int(round(frac ** (1.0 / 3.0) * n)))
    out = np.zeros((n, n, n), dtype=np.uint8)
    out[:e, :e, :e] = 1
    return out
