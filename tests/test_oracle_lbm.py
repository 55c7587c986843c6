"""Pins of the oracle's D3Q19 BGK twoPop pull step:
lattice moments, conservation on a periodic box and in the cavity,
equilibrium fixed point, shear-wave viscous decay against its analytic
rate, z-mirror symmetry, and an independent two-phase (np.roll stream, then
collide) brute force."""
import numpy as np
import pytest

import oracle
import synth

C, W, OPP = oracle.lbm_lattice()


def test_lattice_moments():
    assert abs(W.sum() - 1.0) < 1e-15
    assert np.max(np.abs(W @ C)) < 1e-16
    assert np.max(np.abs(np.einsum("i,ia,ib->ab", W, C, C) - np.eye(3) / 3)) < 3e-16
    d = np.eye(3)
    iso = (np.einsum("ab,cd->abcd", d, d) + np.einsum("ac,bd->abcd", d, d)
           + np.einsum("ad,bc->abcd", d, d)) / 9.0
    assert np.max(np.abs(np.einsum("i,ia,ib,ic,id->abcd", W, C, C, C, C) - iso)) < 3e-16
    assert np.all(C[OPP] == -C)
    assert len({tuple(c) for c in C}) == 19
    # halo-contiguous order: 9..13 have c_z = +1, 14..18 have c_z = -1
    assert np.all(C[9:14, 2] == 1) and np.all(C[14:19, 2] == -1)


def feq(rho, u):
    cu = np.einsum("ia,a...->i...", C.astype(float), u)
    usq = (u * u).sum(0)
    return W[:, None, None, None] * rho * (1 + 3 * cu + 4.5 * cu * cu - 1.5 * usq)


def random_state(shape, seed, amp=0.02):
    nz, ny, nx = shape
    rho = 1.0 + amp * synth.uniform((nx, ny, nz), seed=seed)
    u = amp * synth.uniform((nx, ny, nz), card=3, seed=seed + 1)
    return feq(rho, u) * (1 + 0.01 * synth.uniform((nx, ny, nz), card=19, seed=seed + 2))


def test_equilibrium_moments_return_rho_u():
    f = feq(np.full((3, 4, 5), 1.1), 0.03 * np.ones((3, 3, 4, 5)))
    rho, u = oracle.lbm_macroscopic(f)
    assert np.allclose(rho, 1.1, atol=1e-15) and np.allclose(u, 0.03, atol=1e-15)


def test_periodic_conservation_mass_momentum():
    f = random_state((6, 7, 8), 3)
    m0 = f.sum()
    p0 = np.einsum("ia,izyx->a", C.astype(float), f)
    for _ in range(60):
        f = oracle.lbm_step(f, 1.3, bc=oracle.LBM_PERIODIC)
    assert abs(f.sum() - m0) / m0 < 1e-13
    assert np.max(np.abs(np.einsum("ia,izyx->a", C.astype(float), f) - p0)) < 1e-12


def test_cavity_mass_conserved_with_moving_lid():
    n = 10
    f = np.broadcast_to(W[:, None, None, None], (19, n, n, n)).copy()
    m0 = f.sum()
    for _ in range(100):
        f = oracle.lbm_step(f, oracle.lbm_omega(n), u_lid=0.05)
    assert abs(f.sum() - m0) / m0 < 1e-13
    rho, u = oracle.lbm_macroscopic(f)
    assert 0.005 < np.abs(u[0]).max() < 0.05  # the lid drives a flow
    # the lid moves in +x: the cells under the lid are dragged in +x
    assert u[0, :, -1, :].mean() > 0


def test_uniform_rest_state_is_fixed_point():
    f = np.broadcast_to((1.3 * W)[:, None, None, None], (19, 5, 6, 7)).copy()
    g = oracle.lbm_step(f, 0.9, u_lid=0.0)
    assert np.max(np.abs(g - f)) < 1e-16
    u0 = np.stack([np.full((5, 6, 7), 0.02), np.full((5, 6, 7), -0.01), np.full((5, 6, 7), 0.03)])
    f = feq(np.ones((5, 6, 7)), u0)
    g = oracle.lbm_step(f, 0.9, bc=oracle.LBM_PERIODIC)
    assert np.max(np.abs(g - f)) < 1e-16


def test_cavity_z_mirror_symmetry():
    n = 8
    f = np.broadcast_to(W[:, None, None, None], (19, n, n, n)).copy()
    for _ in range(40):
        f = oracle.lbm_step(f, oracle.lbm_omega(n), u_lid=0.05)
    rho, u = oracle.lbm_macroscopic(f)
    assert np.max(np.abs(u[0] - u[0][::-1])) < 1e-13
    assert np.max(np.abs(u[2] + u[2][::-1])) < 1e-13
    assert np.max(np.abs(rho - rho[::-1])) < 1e-13
    assert np.max(np.abs(u[2])) > 1e-4  # not trivially zero


def test_shear_wave_viscous_decay():
    L, omega, U, steps = 32, 1.2, 1e-3, 400
    y = np.arange(L)
    ux = U * np.sin(2 * np.pi * y / L)
    u = np.zeros((3, 2, L, 2))
    u[0] = ux[None, :, None]
    f = feq(np.ones((2, L, 2)), u)
    for _ in range(steps):
        f = oracle.lbm_step(f, omega, bc=oracle.LBM_PERIODIC)
    _, u = oracle.lbm_macroscopic(f)
    amp = 2.0 / L * np.sum(u[0, 0, :, 0] * np.sin(2 * np.pi * y / L))
    nu = (1 / omega - 0.5) / 3
    ratio = amp / (U * np.exp(-nu * (2 * np.pi / L) ** 2 * steps))
    assert abs(ratio - 1) < 0.01


def brute_two_phase(f, omega, bc, u_lid=0.05):
    """Independent brute force: stream every population with np.roll (push
    form of x - c_i sources), then apply bounce-back by explicit loops, then
    BGK collide with the textbook equilibrium written out here."""
    nz, ny, nx = f.shape[1:]
    g = np.empty_like(f)
    for i in range(19):
        cx, cy, cz = C[i]
        g[i] = np.roll(f[i], shift=(cz, cy, cx), axis=(0, 1, 2))
    if bc == oracle.LBM_CAVITY:
        for i in range(19):
            cx, cy, cz = C[i]
            for z in range(nz):
                for yy in range(ny):
                    for x in range(nx):
                        sx, sy, sz = x - cx, yy - cy, z - cz
                        if 0 <= sx < nx and 0 <= sy < ny and 0 <= sz < nz:
                            continue
                        v = f[OPP[i], z, yy, x]
                        if sy == ny and 0 <= sx < nx and 0 <= sz < nz:
                            v += 6 * W[i] * 1.0 * cx * u_lid
                        g[i, z, yy, x] = v
    rho = g.sum(0)
    u = np.einsum("ia,i...->a...", C.astype(float), g) / rho
    return g - omega * (g - feq(rho, u))


@pytest.mark.parametrize("bc", [oracle.LBM_PERIODIC, oracle.LBM_CAVITY])
def test_brute_force_two_phase_equals_fused_pull(bc):
    f = random_state((4, 5, 6), 11)
    got = oracle.lbm_step(f, 0.8, bc=bc)
    exp = brute_two_phase(f, 0.8, bc)
    assert np.max(np.abs(got - exp) / np.abs(exp)) < 1e-14


# ---- element-sparse domains -----------------------------
def brute_masked(f, omega, bc, active, u_lid=0.05):
    """Independent brute force of the masked step: np.roll streaming of every
    population (periodic images), then, cell by cell, replace populations whose
    source x - c_i is not an active in-box cell by the bounce-back value."""
    nz, ny, nx = f.shape[1:]
    g = np.empty_like(f)
    for i in range(19):
        cx, cy, cz = C[i]
        g[i] = np.roll(f[i], shift=(cz, cy, cx), axis=(0, 1, 2))
    for z in range(nz):
        for yy in range(ny):
            for x in range(nx):
                for i in range(19):
                    cx, cy, cz = C[i]
                    sx, sy, sz = x - cx, yy - cy, z - cz
                    if bc == oracle.LBM_PERIODIC:
                        ok = active[sz % nz, sy % ny, sx % nx]
                        lid = False
                    else:
                        inbox = 0 <= sx < nx and 0 <= sy < ny and 0 <= sz < nz
                        ok = inbox and active[sz, sy, sx]
                        lid = sy == ny and 0 <= sx < nx and 0 <= sz < nz
                    if not ok:
                        v = f[OPP[i], z, yy, x]
                        if lid:
                            v += 6 * W[i] * 1.0 * cx * u_lid
                        g[i, z, yy, x] = v
    rho = g.sum(0)
    u = np.einsum("ia,i...->a...", C.astype(float), g) / rho
    out = g - omega * (g - feq(rho, u))
    return np.where(active[None].astype(bool), out, 0.0)


@pytest.mark.parametrize("bc", [oracle.LBM_PERIODIC, oracle.LBM_CAVITY])
def test_masked_step_equals_brute_force(bc):
    shape = (5, 6, 7)
    f = random_state(shape, 21)
    rng = np.random.default_rng(3)
    active = (rng.random(shape) < 0.7).astype(np.uint8)
    got = oracle.lbm_step(f, 0.9, bc=bc, active=active)
    exp = brute_masked(f, 0.9, bc, active)
    m = active.astype(bool)
    assert np.all(got[:, ~m] == 0.0)
    assert np.max(np.abs(got[:, m] - exp[:, m]) / np.abs(exp[:, m])) < 1e-14


def test_masked_full_mask_is_the_dense_step():
    f = random_state((4, 5, 6), 5)
    for bc in (oracle.LBM_PERIODIC, oracle.LBM_CAVITY):
        assert np.array_equal(oracle.lbm_step(f, 0.8, bc=bc, active=np.ones((4, 5, 6), np.uint8)),
                              oracle.lbm_step(f, 0.8, bc=bc))


def test_closed_sphere_conserves_mass():
    """Half-way bounce-back on stationary walls conserves mass exactly (to
    rounding) in any closed fluid region: a sphere that does not touch the
    lid, 150 steps from a perturbed state."""
    n = 12
    active = synth.sphere_mask(n)
    f = random_state((n, n, n), 7) * active[None]
    m0 = f.sum()
    for _ in range(150):
        f = oracle.lbm_step(f, 1.1, bc=oracle.LBM_CAVITY, active=active)
    assert abs(f.sum() - m0) / m0 < 1e-13
