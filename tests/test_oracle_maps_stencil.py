"""Pins of the oracle's map, reduce and 7-point stencil (SURVEY.md §8(c)
c2-c4, c7, c9) against things other than the oracle itself: exact rational
arithmetic, closed forms, a discrete eigenvector, operator symmetry and a
brute-force dense matrix built from the stencil's definition."""
from fractions import Fraction

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.filterwarnings("ignore")


# ---- maps: PAPER.md eq. L104 -------------------------------------------
def test_axpy_dyadic_exact_vs_rationals():
    x = synth.int_uniform((7, 5, 3), seed=3)
    y = synth.int_uniform((7, 5, 3), seed=4)
    a = 0.125
    got = oracle.axpy(a, x, y)
    exp = np.array([float(Fraction(1, 8) * Fraction(int(u)) + Fraction(int(v)))
                    for u, v in zip(x.ravel(), y.ravel())]).reshape(x.shape)
    assert np.array_equal(got, exp)


def test_axpby_copy_scale_semantics_ignore_y():
    x = synth.uniform((4, 4, 4), seed=1)
    y = np.full_like(x, np.nan)
    assert np.array_equal(oracle.axpby(2.0, x, 0.0, y), 2.0 * x)
    z = oracle.axpby(0.5, x, -3.0, synth.int_uniform((4, 4, 4), seed=9))
    assert np.all(np.isfinite(z))


def test_axpby_real_inputs_within_one_rounding_of_exact():
    x = synth.uniform((6, 5, 4), seed=11)
    y = synth.uniform((6, 5, 4), seed=12)
    a, b = 0.3, -1.7
    got = oracle.axpby(a, x, b, y)
    for g, u, v in zip(got.ravel(), x.ravel(), y.ravel()):
        exact = Fraction(a) * Fraction(float(u)) + Fraction(b) * Fraction(float(v))
        scale = abs(a * u) + abs(b * v)
        assert abs(Fraction(float(g)) - exact) <= Fraction(2.3e-16) * Fraction(scale)


# ---- reduce: PAPER.md eq. L129 -------------------------------------------
def test_dot_integer_exact():
    n = 1 << 16
    idx = np.arange(n)
    x = (idx % 7).astype(np.float64)
    y = (idx % 5).astype(np.float64) - 2.0
    exact = int(np.sum((idx % 7).astype(np.int64) * ((idx % 5).astype(np.int64) - 2)))
    assert oracle.dot(x, y) == float(exact)


def test_dot_is_correctly_rounded_on_cancelling_sums():
    rng = np.random.default_rng(0)
    x = rng.standard_normal(3000) * np.exp(rng.uniform(-20, 20, 3000))
    y = rng.standard_normal(3000)
    # make it ill-conditioned: append the negated products
    x = np.concatenate([x, x, [1e-3]])
    y = np.concatenate([y, -y, [1.0]])
    exact = sum((Fraction(float(a)) * Fraction(float(b)) for a, b in zip(x, y)), Fraction(0))
    got = oracle.dot(x, y)
    assert abs(Fraction(got) - exact) <= abs(exact) * Fraction(1.2e-16)


def test_dot_random_vs_exact_rational():
    x = synth.uniform((13, 11, 9), seed=5).ravel()
    y = synth.uniform((13, 11, 9), seed=6).ravel()
    exact = sum((Fraction(float(a)) * Fraction(float(b)) for a, b in zip(x, y)), Fraction(0))
    assert abs(Fraction(oracle.dot(x, y)) - exact) <= abs(exact) * Fraction(1.2e-16)


# ---- 7-point Laplacian: PAPER.md L145-L152; SURVEY.md §8(c) c3 -----------
def _coords(shape):
    nz, ny, nx = shape
    Z, Y, X = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    return X.astype(np.float64), Y.astype(np.float64), Z.astype(np.float64)


@pytest.mark.parametrize("shape", [(5, 7, 9), (8, 8, 8), (3, 4, 11)])
def test_laplace_quadratic_closed_form_bit_exact(shape):
    """u = X^2+Y^2+Z^2: L u = 6 - sum over missing neighbours of u(ghost),
    evaluated at the ghost coordinate (outside value 0)."""
    X, Y, Z = _coords(shape)
    u = X * X + Y * Y + Z * Z
    nz, ny, nx = shape
    exp = np.full(shape, 6.0)
    for axis_val, n, which in ((X, nx, 0), (Y, ny, 1), (Z, nz, 2)):
        for side, ghost in ((axis_val == 0, -1.0), (axis_val == n - 1, float(n))):
            coords = [X.copy(), Y.copy(), Z.copy()]
            coords[which] = np.full(shape, ghost)
            g = coords[0] ** 2 + coords[1] ** 2 + coords[2] ** 2
            exp = np.where(side, exp - g, exp)
    assert np.array_equal(oracle.laplace7(u), exp)


def test_laplace_outside_value_counts_missing_neighbours():
    shape = (4, 5, 6)
    u = np.zeros(shape)
    c = 2.5
    X, Y, Z = _coords(shape)
    missing = ((X == 0).astype(int) + (X == 5) + (Y == 0) + (Y == 4) + (Z == 0) + (Z == 3))
    assert np.array_equal(oracle.laplace7(u, outside=c), c * missing)


@pytest.mark.parametrize("shape", [(6, 7, 8), (16, 16, 16)])
def test_laplace_discrete_eigenvector(shape):
    nz, ny, nx = shape
    sx = np.sin(np.pi * np.arange(1, nx + 1) / (nx + 1))
    sy = np.sin(np.pi * np.arange(1, ny + 1) / (ny + 1))
    sz = np.sin(np.pi * np.arange(1, nz + 1) / (nz + 1))
    u = sz[:, None, None] * sy[None, :, None] * sx[None, None, :]
    lam = sum(2.0 - 2.0 * np.cos(np.pi / (n + 1)) for n in (nx, ny, nz))
    assert np.max(np.abs(-oracle.laplace7(u) - lam * u)) < 1e-14


def test_laplace_symmetric():
    u = synth.uniform((9, 8, 7), seed=1)
    v = synth.uniform((9, 8, 7), seed=2)
    a = oracle.dot(oracle.laplace7(u), v)
    b = oracle.dot(u, oracle.laplace7(v))
    assert abs(a - b) <= 1e-13 * (abs(a) + 1.0)


def dense_laplacian(shape):
    """Brute force: the matrix of the 7-point operator assembled from its
    definition (-6 on the diagonal, 1 for each face neighbour in the box)."""
    nz, ny, nx = shape
    n = nx * ny * nz
    M = np.zeros((n, n))
    for z in range(nz):
        for y in range(ny):
            for x in range(nx):
                i = x + nx * (y + ny * z)
                M[i, i] = -6.0
                for dx, dy, dz in ((1, 0, 0), (-1, 0, 0), (0, 1, 0), (0, -1, 0), (0, 0, 1), (0, 0, -1)):
                    a, b, c = x + dx, y + dy, z + dz
                    if 0 <= a < nx and 0 <= b < ny and 0 <= c < nz:
                        M[i, a + nx * (b + ny * c)] = 1.0
    return M


def test_laplace_brute_force_8cubed():
    shape = (8, 8, 8)
    M = dense_laplacian(shape)
    x = synth.uniform((8, 8, 8), seed=7)
    got = oracle.laplace7(x).ravel()
    exp = M @ x.ravel()
    s = np.abs(M) @ np.abs(x.ravel())
    assert np.max(np.abs(got - exp) / s) < 4e-16
    ev = np.linalg.eigvalsh(-M)
    assert abs(ev[0] - 3 * (2 - 2 * np.cos(np.pi / 9))) < 1e-12  # lambda_min = 0.3618


# ---- element-sparse stencil: PAPER.md L248; SURVEY.md §8(c) c7 -----------
def test_sparse_full_mask_equals_dense_bitwise():
    x = synth.uniform((9, 7, 5), seed=3)
    m = np.ones(x.shape, dtype=np.uint8)
    assert np.array_equal(oracle.sparse_laplace7(m, x), oracle.laplace7(x))


def test_sparse_equals_dense_on_masked_field():
    x = synth.uniform((12, 12, 12), seed=3)
    m = synth.sphere_mask(12, 0.45)
    assert 0 < m.sum() < m.size
    xm = np.where(m, x, 0.0)
    exp = np.where(m, oracle.laplace7(xm), 0.0)
    assert np.array_equal(oracle.sparse_laplace7(m, x), exp)


def test_sparse_brute_force_masked_matrix():
    shape = (6, 6, 6)
    m = synth.sphere_mask(6, 0.45).ravel().astype(bool)
    M = dense_laplacian(shape)
    Ms = M[np.ix_(m, m)]
    x = synth.uniform(shape, seed=8)
    got = oracle.sparse_laplace7(m.reshape(shape), x).ravel()
    assert np.max(np.abs(got[m] - Ms @ x.ravel()[m])) < 1e-14
    assert np.all(got[~m] == 0.0)


# ---- config C1 loop: Fig. 4a; SURVEY.md §8(c) c9 -------------------------
def test_c1_loop_exact_regime_vs_rationals():
    shape = (4, 5, 6)
    nz, ny, nx = shape
    x0 = synth.int_uniform((nx, ny, nz), seed=1)
    xo, yo, dots = oracle.c1_loop(x0, a=0.125, iters=10)
    M = dense_laplacian(shape).astype(np.int64)
    a = Fraction(1, 8)
    x = [Fraction(int(v)) for v in x0.ravel()]
    y = [Fraction(0)] * len(x)
    nbrs = [np.nonzero(M[i])[0] for i in range(len(x))]
    exact_dots = []
    for _ in range(10):
        x = [xi + a * yi for xi, yi in zip(x, y)]
        y = [sum((M[i, j] * x[j] for j in nbrs[i]), Fraction(0)) for i in range(len(x))]
        exact_dots.append(sum((xi * yi for xi, yi in zip(x, y)), Fraction(0)))
    assert np.array_equal(xo.ravel(), np.array([float(v) for v in x]))
    assert np.array_equal(yo.ravel(), np.array([float(v) for v in y]))
    for d, e in zip(dots, exact_dots):
        assert abs(Fraction(float(d)) - e) <= abs(e) * Fraction(1.2e-16)


def test_sphere_occupancy_config_c4():
    """C4 domain at N = 512: the lattice count of cell centres inside the
    sphere r = 0.41528 N matches the continuous volume 4/3 pi r^3 to 1e-4
    (and is 30.00 % of the box).  SURVEY.md quotes 40,265,544 from a scratch
    run; the definition in synth.sphere_mask gives 40,263,912 — DESIGN.md
    "Readings" records that the survey figure was not reproducible."""
    m = synth.sphere_mask(512)
    cnt = int(m.sum(dtype=np.int64))
    vol = 4.0 / 3.0 * np.pi * (0.41528 * 512) ** 3
    assert abs(cnt - vol) / vol < 1e-4
    assert round(cnt / 512 ** 3, 4) == 0.3
