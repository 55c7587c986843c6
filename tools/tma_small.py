import sys; sys.path.insert(0, '.')
import paper_conf_ipps_meneghinmjm22_b200 as nb
g = nb.Grid((64, 64, 64))
b, x = nb.Field(g), nb.Field(g)
b.fill(nb.FILL_POISSON_RHS); x.fill_const(0.0)
r = nb.nb_cg_solve(x, b, max_iter=3)
print("ok", r.iters)
