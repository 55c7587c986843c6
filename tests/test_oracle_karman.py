"""Pins of the oracle's D2Q9 step (the 2-D Kármán vortex
street of PAPER.md Table I): lattice moments, the uniform inflow as an exact
fixed point of the channel, mass conservation with a bounce-back cylinder
in a periodic box, and an independent np.roll brute force of the pull step
with the inflow / outflow / bounce-back readings."""
import numpy as np
import pytest

import oracle
import synth

C, W, OPP = oracle.d2q9_lattice()


def feq(rho, ux, uy):
    cu = C[:, 0, None, None] * ux + C[:, 1, None, None] * uy
    return W[:, None, None] * rho * (1 + 3 * cu + 4.5 * cu * cu - 1.5 * (ux * ux + uy * uy))


def test_d2q9_moments():
    assert abs(W.sum() - 1) < 1e-16
    assert np.max(np.abs(W @ C)) < 1e-16
    assert np.max(np.abs(np.einsum("i,ia,ib->ab", W, C, C) - np.eye(2) / 3)) < 1e-16
    assert np.all(C[OPP] == -C)


def test_uniform_inflow_is_a_fixed_point_of_the_empty_channel():
    nx, ny, u = 24, 10, 0.08
    f = feq(np.ones((ny, nx)), np.full((ny, nx), u), np.zeros((ny, nx)))
    g = f
    for _ in range(20):
        g = oracle.d2q9_step(g, 1.7, u, (0, 0, -1))
    assert np.max(np.abs(g - f)) < 1e-15


def test_periodic_box_with_cylinder_conserves_mass():
    nx, ny = 20, 16
    rho = 1 + 0.05 * synth.uniform((nx, ny, 1), seed=3)[0]
    ux = 0.05 * synth.uniform((nx, ny, 1), seed=4)[0]
    uy = 0.05 * synth.uniform((nx, ny, 1), seed=5)[0]
    cyl = (8, 7, 3)
    yy, xx = np.mgrid[0:ny, 0:nx]
    solid = (xx - 8) ** 2 + (yy - 7) ** 2 <= 9
    f = feq(rho, ux, uy) * ~solid
    m0 = f.sum()
    for _ in range(200):
        f = oracle.d2q9_step(f, 1.3, 0.0, cyl, bc=oracle.D2Q9_PERIODIC)
    assert np.all(f[:, solid] == 0)
    assert abs(f.sum() - m0) / m0 < 1e-13


def brute(f, omega, u_in, cyl, bc):
    """np.roll streaming (push form), then the boundary readings cell by
    cell, then the textbook BGK collision."""
    _, ny, nx = f.shape
    cx, cy, r = cyl
    yy, xx = np.mgrid[0:ny, 0:nx]
    solid = (xx - cx) ** 2 + (yy - cy) ** 2 <= r * r if r >= 0 else np.zeros((ny, nx), bool)
    g = np.stack([np.roll(f[i], shift=(C[i, 1], C[i, 0]), axis=(0, 1)) for i in range(9)])
    fin_eq = feq(np.ones((1, 1)), np.full((1, 1), u_in), np.zeros((1, 1)))[:, 0, 0]
    for y in range(ny):
        for x in range(nx):
            for i in range(9):
                sx, sy = x - C[i, 0], (y - C[i, 1]) % ny
                if bc == oracle.D2Q9_PERIODIC:
                    sx %= nx
                elif sx < 0:
                    g[i, y, x] = fin_eq[i]
                    continue
                elif sx >= nx:
                    sx = nx - 1
                if solid[sy, sx]:
                    g[i, y, x] = f[OPP[i], y, x]
                else:
                    g[i, y, x] = f[i, sy, sx]
    rho = g.sum(0)
    ux = (C[:, 0, None, None] * g).sum(0) / rho
    uy = (C[:, 1, None, None] * g).sum(0) / rho
    out = g - omega * (g - feq(rho, ux, uy))
    return np.where(solid[None], 0.0, out)


@pytest.mark.parametrize("bc", [oracle.D2Q9_CHANNEL, oracle.D2Q9_PERIODIC])
def test_brute_force(bc):
    nx, ny = 13, 9
    rho = 1 + 0.05 * synth.uniform((nx, ny, 1), seed=6)[0]
    ux = 0.06 + 0.02 * synth.uniform((nx, ny, 1), seed=7)[0]
    uy = 0.02 * synth.uniform((nx, ny, 1), seed=8)[0]
    f = feq(rho, ux, uy)
    got = oracle.d2q9_step(f, 1.6, 0.06, (4, 4, 2), bc=bc)
    exp = brute(f, 1.6, 0.06, (4, 4, 2), bc)
    assert np.max(np.abs(got - exp)) < 1e-15
