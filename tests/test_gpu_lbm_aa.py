"""AA-pattern LBM: one population buffer updated in
place.  The gathered populations and the collision are twoPop's, so an even
number of AA steps must equal the same number of twoPop steps bit for bit —
cavity (walls + moving lid) and periodic boxes, one and several partitions
(the odd steps' stores into the neighbours' boundary planes) — and agree
with the oracle."""
import numpy as np
import pytest

import oracle
import paper_conf_ipps_meneghinmjm22_b200 as nb
import synth

pytestmark = pytest.mark.gpu
C, W, OPP = oracle.lbm_lattice()


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__
    __graft_entry__.build()
    assert nb.nb_device_count() > 0


def state(dims, seed):
    rho = 1.0 + 0.02 * synth.uniform(dims, seed=seed)
    u = 0.02 * synth.uniform(dims, card=3, seed=seed + 1)
    cu = np.einsum("ia,a...->i...", C.astype(float), u)
    f = W[:, None, None, None] * rho * (1 + 3 * cu + 4.5 * cu * cu - 1.5 * (u * u).sum(0))
    return (f * (1 + 0.01 * synth.uniform(dims, card=19, seed=seed + 2))).astype(np.float32)


def run(dims, parts, f0, steps, bc, aa, omega=0.85):
    with nb.Grid(dims, nparts=parts, devices=[0] * parts) as g:
        a, b = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
        a.upload(f0)
        if aa:
            nb.nb_lbm_step_aa(a, omega, steps, bc=bc)
        else:
            a, b = nb.nb_lbm_step(a, b, omega, steps, bc=bc, occ=nb.OCC_NONE)
        out = a.download()
        a.close(), b.close()
    return out


@pytest.mark.parametrize("bc", [nb.LBM_CAVITY, nb.LBM_PERIODIC])
@pytest.mark.parametrize("parts", [1, 3])
def test_aa_equals_twopop_bitwise(bc, parts):
    dims = (22, 17, 15)
    f0 = state(dims, 4)
    for steps in (2, 8):
        assert np.array_equal(run(dims, parts, f0, steps, bc, True), run(dims, parts, f0, steps, bc, False)), steps


def test_aa_two_steps_vs_oracle():
    dims = (16, 14, 12)
    f0 = state(dims, 7)
    got = run(dims, 2, f0, 2, nb.LBM_CAVITY, True)
    e = oracle.lbm_step(oracle.lbm_step(f0, 0.85), 0.85)
    assert np.max(np.abs(got - e) / np.abs(e)) <= 2e-5


def test_aa_rejects_odd_steps():
    with nb.Grid((8, 8, 8)) as g:
        a = nb.Field(g, "f32", 19)
        with pytest.raises(nb.NbError):
            nb.nb_lbm_step_aa(a, 0.9, 3)
        a.close()
