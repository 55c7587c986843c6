"""Short driver for ncu captures: a few CG iterations and LBM steps at the
bench sizes (512^3), eager launches (no graphs) so each kernel is visible."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["NB_NO_GRAPH"] = "1"
import paper_conf_ipps_meneghinmjm22_b200 as nb  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
what = sys.argv[2] if len(sys.argv) > 2 else "cg,lbm"
if "cg" in what:
    g = nb.Grid((n, n, n))
    b, x = nb.Field(g), nb.Field(g)
    b.fill(nb.FILL_POISSON_RHS)
    x.fill_const(0.0)
    cg = nb.CG(x, b)
    cg.iterate(3)
    cg.finish()
    cg.close()
    b.close(), x.close()
    g.close()
if "lbm" in what:
    g = nb.Grid((n, n, n))
    fa, fb = nb.Field(g, "f32", 19), nb.Field(g, "f32", 19)
    nb.nb_lbm_init(fa, 1.0, (0, 0, 0))
    fa, fb = nb.nb_lbm_step(fa, fb, 0.7886, 3)
    g.sync()
    fa.close(), fb.close()
    g.close()
if "sparse" in what:
    import synth
    m = synth.sphere_mask(n)
    g = nb.Grid((n, n, n), active=m)
    b, x = nb.Field(g), nb.Field(g)
    b.fill_uniform(seed=4)
    x.fill_const(0.0)
    cg = nb.CG(x, b)
    cg.iterate(3)
    cg.finish()
    cg.close()
    b.close(), x.close()
    g.close()
if "fem" in what:
    nf = min(n, 384)
    g = nb.Grid((nf, nf, nf))
    b, x = nb.Field(g, card=3), nb.Field(g, card=3)
    nb.nb_fem27_rhs(b, 1.0)
    x.fill_const(0.0)
    cg = nb.CG(x, b, op=nb.OP_FEM27)
    cg.iterate(3)
    cg.finish()
    cg.close()
    b.close(), x.close()
    g.close()
if "spfem" in what:  # FEM on an element-sparse sphere
    import synth
    nf = min(n, 384)
    g = nb.Grid((nf, nf, nf), active=synth.sphere_mask(nf))
    b, x = nb.Field(g, card=3), nb.Field(g, card=3)
    nb.nb_fem27_rhs(b, 1.0)
    x.fill_const(0.0)
    cg = nb.CG(x, b, op=nb.OP_FEM27)
    cg.iterate(2)
    cg.finish()
    cg.close()
    b.close(), x.close()
    g.close()
print("prof driver done")
