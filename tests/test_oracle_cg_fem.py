"""Pins of the oracle's CG and FEM operator (c8)
against the analytic manufactured solution, a discrete eigenvector, a dense
direct solve, analytic element-stiffness entries, rigid-body modes, the
patch test and the strain-energy closed form."""
import numpy as np
import pytest

import oracle
import synth

from test_oracle_maps_stencil import dense_laplacian


# ---- CG on A = -L ------------------------------------
@pytest.mark.parametrize("n,max_it", [(16, 60), (24, 90)])
def test_cg_manufactured_solution_converges_to_analytic(n, max_it):
    b = synth.poisson_poly_rhs((n, n, n))
    ustar = synth.poisson_poly_solution(n)
    # u* is exactly the discrete solution: A u* = b (operator exact on quadratics)
    assert np.max(np.abs(-oracle.laplace7(ustar) - b)) < 16 * 2.3e-16 * np.max(np.abs(ustar))
    x, res, hist = oracle.cg(b, max_iter=max_it, rtol=1e-12)
    assert res.converged == 1
    assert res.iters < 3.2 * n
    assert np.max(np.abs(x - ustar)) < 5e-14


def test_cg_single_eigenvector_one_iteration():
    n = 12
    s = np.sin(np.pi * np.arange(1, n + 1) / (n + 1))
    u = s[:, None, None] * s[None, :, None] * s[None, None, :]
    lam = 3 * (2 - 2 * np.cos(np.pi / (n + 1)))
    x, res, _ = oracle.cg(lam * u, max_iter=5, rtol=1e-13)
    assert res.iters == 1
    assert np.max(np.abs(x - u)) < 1e-14


def test_cg_dense_direct_solve_8cubed():
    shape = (8, 8, 8)
    A = -dense_laplacian(shape)
    b = synth.uniform(shape, seed=2)
    xd = np.linalg.solve(A, b.ravel())
    x, res, hist = oracle.cg(b, max_iter=60, rtol=0.0)
    assert np.max(np.abs(x.ravel() - xd)) < 1e-13
    # recursive residual tracks the true residual
    rtrue = b.ravel() - A @ x.ravel()
    assert abs(np.dot(rtrue, rtrue) - hist[-1]) < 1e-20 + 1e-6 * hist[-1]


def test_cg_residual_history_monotone_in_energy_norm():
    shape = (10, 9, 8)
    A = -dense_laplacian(shape)
    b = synth.uniform(shape[::-1], seed=3)
    xd = np.linalg.solve(A, b.ravel())
    errs = []
    for k in range(1, 16, 2):
        x, res, _ = oracle.cg(b, max_iter=k)
        e = x.ravel() - xd
        errs.append(e @ A @ e)
    assert errs[-1] > 1e-24
    assert all(a > b for a, b in zip(errs, errs[1:]))


def test_cg_zero_rhs_is_zero_iterations():
    x, res, _ = oracle.cg(np.zeros((4, 4, 4)), max_iter=5, rtol=1e-8)
    assert res.iters == 0 and res.converged == 2 and np.all(x == 0)


def test_sparse_cg_full_mask_reproduces_dense_bitwise():
    b = synth.uniform((6, 7, 8), seed=4)
    m = np.ones(b.shape, dtype=np.uint8)
    x1, r1, h1 = oracle.cg(b, max_iter=20)
    x2, r2, h2 = oracle.cg(b, max_iter=20, op=oracle.OP_SPARSE7, mask=m)
    assert np.array_equal(x1, x2) and np.array_equal(h1, h2)


def test_sparse_cg_vs_direct_on_sphere():
    n = 8
    m = synth.sphere_mask(n, 0.45)
    act = m.ravel().astype(bool)
    A = -dense_laplacian((n, n, n))[np.ix_(act, act)]
    b = np.where(m, synth.uniform((n, n, n), seed=5), 0.0)
    x, res, _ = oracle.cg(b, max_iter=80, op=oracle.OP_SPARSE7, mask=m, rtol=1e-14)
    xd = np.linalg.solve(A, b.ravel()[act])
    assert np.max(np.abs(x.ravel()[act] - xd)) < 1e-12
    assert np.all(x.ravel()[~act] == 0.0)


# ---- FEM -------------------------
E, NU = 1.0, 0.3
LAM = E * NU / ((1 + NU) * (1 - 2 * NU))
MU = E / (2 * (1 + NU))


def test_ke_analytic_entries():
    ke = oracle.fem_ke(E, NU)
    # K[0,0] = (lam + 4 mu) * int (dN0/dx)^2 = (lam + 4 mu)/9  (= 0.235043)
    assert abs(ke[0, 0] - (LAM + 4 * MU) / 9) < 1e-15
    assert abs(ke[0, 0] - 0.2350427350427350) < 1e-15
    # K[0,1] (node 0 x-dof, node 0 y-dof) = (lam + mu) * int dN0/dx dN0/dy = (lam+mu)/12
    assert abs(ke[0, 1] - (LAM + MU) / 12) < 1e-15
    # node 0 x-dof vs node 1 (the +x neighbour) x-dof: (lam+2mu) int dN0x dN1x + mu (int dN0y dN1y + dN0z dN1z)
    #   int dN0x dN1x = -1/9 ; int dN0y dN1y = int (1-x)x (1-z)^2 = 1/6 * 1/3 ... = 1/18 each
    assert abs(ke[0, 3] - (-(LAM + 2 * MU) / 9 + MU * (1 / 18 + 1 / 18))) < 1e-15


def test_ke_symmetric_with_six_rigid_modes():
    ke = oracle.fem_ke(E, NU)
    assert np.max(np.abs(ke - ke.T)) < 1e-16
    ev = np.linalg.eigvalsh(ke)
    assert np.all(np.abs(ev[:6]) < 1e-14) and ev[6] > 1e-2
    # explicit rigid modes: 3 translations + 3 rotations about the centre
    pts = np.array([[a & 1, (a >> 1) & 1, (a >> 2) & 1] for a in range(8)], dtype=float) - 0.5
    modes = []
    for d in range(3):
        m = np.zeros((8, 3)); m[:, d] = 1; modes.append(m.ravel())
    for axis in np.eye(3):
        modes.append(np.cross(axis, pts).ravel())
    for m in modes:
        assert np.max(np.abs(ke @ m)) < 1e-15


def test_ke_uniform_strain_energy_closed_form():
    """u = G x on one element: u^T K_e u = eps^T D eps (unit volume)."""
    ke = oracle.fem_ke(E, NU)
    rng = np.random.default_rng(1)
    G = rng.standard_normal((3, 3))
    pts = np.array([[a & 1, (a >> 1) & 1, (a >> 2) & 1] for a in range(8)], dtype=float)
    u = (pts @ G.T).ravel()
    eps = np.array([G[0, 0], G[1, 1], G[2, 2], G[0, 1] + G[1, 0], G[1, 2] + G[2, 1], G[2, 0] + G[0, 2]])
    D = np.zeros((6, 6)); D[:3, :3] = LAM; D[np.arange(3), np.arange(3)] += 2 * MU
    D[np.arange(3, 6), np.arange(3, 6)] = MU
    assert abs(u @ ke @ u - eps @ D @ eps) < 1e-13


def test_fem_patch_test_and_rigid_motion_on_grid():
    n = 5
    Z, Y, X = np.meshgrid(np.arange(n), np.arange(n), np.arange(n), indexing="ij")
    G = np.array([[0.3, -0.2, 0.1], [0.05, 0.4, -0.3], [0.2, 0.1, -0.1]])
    u = np.stack([G[i, 0] * X + G[i, 1] * Y + G[i, 2] * Z for i in range(3)]).astype(float)
    y = oracle.fem_apply(u, E, NU, dirichlet_z0=False)
    inner = (slice(None), slice(1, -1), slice(1, -1), slice(1, -1))
    assert np.max(np.abs(y[inner])) < 1e-14         # linear field: no interior force
    assert np.max(np.abs(y.reshape(3, -1).sum(1))) < 1e-13  # equilibrium
    # rigid rotation about z: u = (-y, x, 0) -> K u = 0 everywhere
    rot = np.stack([-Y, X, 0 * X]).astype(float)
    assert np.max(np.abs(oracle.fem_apply(rot, E, NU, dirichlet_z0=False))) < 1e-13


def test_fem_brute_force_assembled_matrix():
    """Dense K assembled here from K_e (independent loop) vs matrix-free apply."""
    n = 4
    ke = oracle.fem_ke(E, NU)
    N = n ** 3
    K = np.zeros((3 * N, 3 * N))
    for ez in range(n - 1):
        for ey in range(n - 1):
            for ex in range(n - 1):
                dofs = []
                for a in range(8):
                    i, j, k = ex + (a & 1), ey + ((a >> 1) & 1), ez + ((a >> 2) & 1)
                    node = i + n * (j + n * k)
                    dofs += [d * N + node for d in range(3)]
                K[np.ix_(dofs, dofs)] += ke
    fixed = np.zeros(3 * N, dtype=bool)
    for d in range(3):
        fixed[d * N: d * N + n * n] = True  # z = 0 plane
    Kd = K.copy()
    Kd[fixed, :] = 0; Kd[:, fixed] = 0; Kd[fixed, fixed] = 1
    u = synth.uniform((n, n, n), card=3, seed=9)
    y = oracle.fem_apply(u, E, NU, dirichlet_z0=True)
    assert np.max(np.abs(y.ravel() - Kd @ u.ravel())) < 1e-14
    # 27-point structure: an interior node couples to exactly 27 nodes
    mid = 1 + n * (1 + n * 1)
    cols = np.nonzero(np.abs(K[mid]) > 1e-15)[0] % N
    assert len(set(cols.tolist())) == 27
    # RHS: total load = p * area of the top face
    b = oracle.fem_rhs((n, n, n), 1.0)
    assert abs(b[2].sum() - (n - 1) ** 2) < 1e-14 and np.all(b[:2] == 0)
    # FEM CG solves K u = b
    x, res, _ = oracle.cg(b, max_iter=400, rtol=1e-13, op=oracle.OP_FEM27)
    assert res.converged == 1
    assert np.max(np.abs(Kd @ x.ravel() - b.ravel())) < 1e-11
    assert np.allclose(x.ravel(), np.linalg.solve(Kd, b.ravel()), atol=1e-10)


# ---- Neumann load placement ("the z = N-1 plane had outward
# pressure"; consistent nodal loads, tributary areas
# 1 / 1/2 / 1/4) ------------------------------------------------------------
@pytest.mark.parametrize("dims,dirichlet", [((5, 5, 5), True), ((6, 4, 3), True), ((6, 4, 3), False),
                                            ((4, 5, 2), True)])
def test_fem_rhs_exact_tributary_loads_on_top_plane(dims, dirichlet):
    """b is zero except b_z on the top node plane z = Nz-1, where it is p at
    interior nodes, p/2 on edges and p/4 at corners (dyadic: bit-exact).
    A load on plane Nz-2, on an element's bottom nodes or in x/y fails."""
    nx, ny, nz = dims
    p = 3.0
    b = oracle.fem_rhs(dims, p, dirichlet_z0=dirichlet)
    assert np.all(b[0] == 0) and np.all(b[1] == 0)
    assert np.all(b[2, :nz - 1] == 0)
    ex = np.where((np.arange(nx) == 0) | (np.arange(nx) == nx - 1), 0.5, 1.0)
    ey = np.where((np.arange(ny) == 0) | (np.arange(ny) == ny - 1), 0.5, 1.0)
    expect = p * ey[:, None] * ex[None, :]  # [y][x] tributary area of the top face
    assert np.array_equal(b[2, nz - 1], expect)


def test_fem_rhs_virtual_work_on_stepped_mask():
    """Consistent loads integrate every bilinear test function v(x, y, z)
    exactly over the loaded faces: sum_a b_a v_a = p * sum_faces int v dA.
    On a two-level step (columns x >= 3 cut at z = 2) the exposed top faces
    are the upper plateau at z = 4 and the lower one at z = 2; v = z fixes
    the plane of every face, v = x, y, x*y its position."""
    nx, ny, nz = 6, 4, 5
    mask = np.ones((nz, ny, nx), dtype=np.uint8)
    mask[3:, :, 4:] = 0  # nodes x >= 4 exist only up to z = 2 -> elements ex >= 3 stop at ez = 1
    p = 1.0
    b = oracle.fem_rhs((nx, ny, nz), p, mask=mask)
    assert np.all(b[:2] == 0)
    zz, yy, xx = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    # exposed faces: [ex0, ex1) x [0, ny-1) at height z (analytic integrals of v over unit squares)
    faces = [(0, 3, 4.0), (3, 5, 2.0)]

    def integral(fn):
        tot = 0.0
        for x0, x1, z in faces:
            for ex_ in range(x0, x1):
                for ey_ in range(ny - 1):
                    tot += fn(ex_, ey_, z)
        return tot
    tests = {
        "1": (np.ones_like(xx, dtype=float), lambda x, y, z: 1.0),
        "z": (zz.astype(float), lambda x, y, z: z),
        "x": (xx.astype(float), lambda x, y, z: x + 0.5),
        "y": (yy.astype(float), lambda x, y, z: y + 0.5),
        "xy": ((xx * yy).astype(float), lambda x, y, z: (x + 0.5) * (y + 0.5)),
        "xz": ((xx * zz).astype(float), lambda x, y, z: (x + 0.5) * z),
    }
    for name, (v, fn) in tests.items():
        assert abs(float(np.sum(b[2] * v)) - p * integral(fn)) < 1e-12, name


# ---- FEM on element-sparse domains (
# DESIGN reading 10: an element exists iff its 8 nodes are active) ----------
def _masked_dense_K(mask, ke):
    """K assembled here (numpy scatter, independent of the oracle's element
    loop) over the elements whose 8 nodes are all active."""
    nz, ny, nx = mask.shape
    N = nx * ny * nz
    K = np.zeros((3 * N, 3 * N))
    for ez in range(nz - 1):
        for ey in range(ny - 1):
            for ex in range(nx - 1):
                if not mask[ez:ez + 2, ey:ey + 2, ex:ex + 2].all():
                    continue
                dofs = []
                for a in range(8):
                    i, j, k = ex + (a & 1), ey + ((a >> 1) & 1), ez + ((a >> 2) & 1)
                    node = i + nx * (j + ny * k)
                    dofs += [d * N + node for d in range(3)]
                K[np.ix_(dofs, dofs)] += ke
    return K


def test_fem_masked_apply_brute_force_and_rigid_modes():
    """The masked matrix-free K u equals the brute-force assembly over the
    existing elements (with and without the Dirichlet plane), and on a mask
    with holes rigid translations / a rotation give K u = 0 without
    Dirichlet; nodes in no element get y = 0."""
    rng = np.random.default_rng(11)
    nz, ny, nx = 5, 4, 6
    mask = (rng.random((nz, ny, nx)) < 0.8).astype(np.uint8)
    mask[:, 1:3, 1:4] = 1  # a solid core so that elements exist
    ke = oracle.fem_ke(E, NU)
    K = _masked_dense_K(mask, ke)
    N = nx * ny * nz
    u = synth.uniform((nx, ny, nz), card=3, seed=4) * mask[None]
    y = oracle.fem_apply(u, E, NU, mask=mask, dirichlet_z0=False)
    assert np.max(np.abs(y.ravel() - K @ u.ravel())) < 1e-14
    # Dirichlet z = 0: identity rows / columns on the ACTIVE z = 0 nodes
    fixed = np.zeros(3 * N, dtype=bool)
    act0 = np.zeros((nz, ny, nx), bool)
    act0[0] = mask[0].astype(bool)
    for d in range(3):
        fixed[d * N:(d + 1) * N] = act0.ravel()
    Kd = K.copy()
    Kd[fixed, :] = 0
    Kd[:, fixed] = 0
    Kd[fixed, fixed] = 1
    yd = oracle.fem_apply(u, E, NU, mask=mask, dirichlet_z0=True)
    assert np.max(np.abs(yd.ravel() - Kd @ u.ravel())) < 1e-14
    # rigid modes on the masked body (no Dirichlet)
    Z, Y, X = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    for mode in (np.stack([np.ones_like(X), 0 * X, 0 * X]), np.stack([0 * X, np.ones_like(X), 0 * X]),
                 np.stack([-Y, X, 0 * X])):
        assert np.max(np.abs(oracle.fem_apply(mode.astype(float), E, NU, mask=mask, dirichlet_z0=False))) < 1e-13
    # nodes in no existing element: y = 0
    in_elem = np.zeros((nz, ny, nx), bool)
    for ez in range(nz - 1):
        for ey in range(ny - 1):
            for ex in range(nx - 1):
                if mask[ez:ez + 2, ey:ey + 2, ex:ex + 2].all():
                    in_elem[ez:ez + 2, ey:ey + 2, ex:ex + 2] = True
    lonely = ~in_elem
    assert lonely.any() and np.all(y[:, lonely] == 0)
