/*
 * oracle.c — plain, slow, obviously-correct CPU oracle for the Neon
 * map-stencil hot path (Meneghin et al., "Neon", IPDPS 2022; PAPER.md).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or constant with the CUDA path under
 * paper_conf_ipps_meneghinmjm22_b200/ and never calls it.
 *
 * Rules:
 *   - fp64 everywhere, IEEE round-to-nearest; built with -O2
 *     -ffp-contract=off -fno-fast-math, so no expression is contracted;
 *     the only fma() calls are the explicit error-free TwoProduct in the
 *     reference dot product.
 *   - data in the dense host logical view:
 *     index(c,x,y,z) = x + nx*(y + ny*(z + nz*c)), x fastest.
 *   - loops in natural (z, y, x) order; OpenMP only splits independent
 *     cells across threads, never reorders any per-cell arithmetic.
 *     Reductions keep a fixed order independent of the thread count.
 *
 * Each function cites the passage it follows.  Pins: tests/test_oracle_*.py.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#ifdef _OPENMP
#include <omp.h>
#endif

#define IDX(x, y, z) ((int64_t)(x) + (int64_t)nx * ((int64_t)(y) + (int64_t)ny * (int64_t)(z)))

int or_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

void or_set_num_threads(int n) {
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}

/* ---------------------------------------------------------------------- */
/* Map operations: PAPER.md §III-b eq. L104, "AXPY, copying a Field to     */
/* another, and scaling a Field by a constant" (L107-L108).                */
/* ---------------------------------------------------------------------- */

/* y[i] <- a*x[i] + y[i]  (two roundings: product, then sum) */
void or_axpy(int64_t n, double a, const double *x, double *y) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        double t = a * x[i];
        y[i] = t + y[i];
    }
}

/* y[i] <- a*x[i] + b*y[i]; b == 0 means copy/scale semantics: y is not read
 * (SURVEY.md §8(c) c2 reading). */
void or_axpby(int64_t n, double a, const double *x, double b, double *y) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        double t = a * x[i];
        if (b == 0.0) {
            y[i] = t;
        } else {
            double u = b * y[i];
            y[i] = t + u;
        }
    }
}

/* ---------------------------------------------------------------------- */
/* Reduce: PAPER.md §III-b eq. L129 (dot product, L2 norm), index range   */
/* [0, K) as in L104/L119.  The reference value is the (nearly) correctly  */
/* rounded sum: double-double accumulation (TwoProduct via fma + TwoSum),  */
/* per z-plane, planes combined in increasing z, all in double-double.     */
/* ---------------------------------------------------------------------- */

static inline void two_sum(double a, double b, double *s, double *e) {
    double x = a + b;
    double bv = x - a;
    double av = x - bv;
    *s = x;
    *e = (a - av) + (b - bv);
}

static inline void dd_add(double *hi, double *lo, double v) {
    double s, e;
    two_sum(*hi, v, &s, &e);
    e += *lo;
    two_sum(s, e, hi, lo);
}

static inline void dd_add_prod(double *hi, double *lo, double a, double b) {
    double p = a * b;
    double pe = fma(a, b, -p); /* exact error of the product */
    dd_add(hi, lo, p);
    dd_add(hi, lo, pe);
}

/* n = plane * nplanes.  Double-double sum of x.y into (*ohi, *olo). */
static void dot_planes_dd(int64_t plane, int64_t nplanes, const double *x, const double *y,
                          double *ohi, double *olo) {
    double *phi = (double *)malloc(sizeof(double) * (size_t)(nplanes > 0 ? nplanes : 1));
    double *plo = (double *)malloc(sizeof(double) * (size_t)(nplanes > 0 ? nplanes : 1));
    #pragma omp parallel for schedule(static)
    for (int64_t z = 0; z < nplanes; ++z) {
        double hi = 0.0, lo = 0.0;
        const double *xp = x + z * plane, *yp = y + z * plane;
        for (int64_t i = 0; i < plane; ++i) dd_add_prod(&hi, &lo, xp[i], yp[i]);
        phi[z] = hi;
        plo[z] = lo;
    }
    double hi = 0.0, lo = 0.0;
    for (int64_t z = 0; z < nplanes; ++z) {
        dd_add(&hi, &lo, phi[z]);
        dd_add(&hi, &lo, plo[z]);
    }
    free(phi);
    free(plo);
    *ohi = hi;
    *olo = lo;
}

/* Returns the double-double sum rounded to double. */
double or_dot_planes(int64_t plane, int64_t nplanes, const double *x, const double *y) {
    double hi, lo;
    dot_planes_dd(plane, nplanes, x, y, &hi, &lo);
    return hi + lo;
}

double or_dot(int64_t n, const double *x, const double *y) {
    /* split into 4096-element chunks only to parallelise; the double-double
     * result does not depend on the split beyond ~1e-30 relative. */
    int64_t plane = 4096;
    int64_t full = n / plane;
    double hi, lo;
    dot_planes_dd(plane, full, x, y, &hi, &lo);
    for (int64_t i = full * plane; i < n; ++i) dd_add_prod(&hi, &lo, x[i], y[i]);
    return hi + lo;
}

/* ---------------------------------------------------------------------- */
/* Stencil: 7-point Laplacian (Listing 2 — code lost in */
/* extraction; textbook operator):                    */
/*   L(x)_i = sum_{6 face neighbours j} x_j - 6 x_i                        */
/* A neighbour outside the domain reads outsideDomainValue (L58-L63).      */
/* Summation order: -x, +x, -y, +y, -z, +z, then minus 6*x_i.              */
/* ---------------------------------------------------------------------- */

static inline double nbr(const double *x, int nx, int ny, int nz, int i, int j, int k,
                         double outside) {
    if (i < 0 || i >= nx || j < 0 || j >= ny || k < 0 || k >= nz) return outside;
    return x[IDX(i, j, k)];
}

void or_laplace7(int nx, int ny, int nz, double outside, const double *x, double *y) {
    #pragma omp parallel for schedule(static)
    for (int k = 0; k < nz; ++k)
        for (int j = 0; j < ny; ++j)
            for (int i = 0; i < nx; ++i) {
                double s = nbr(x, nx, ny, nz, i - 1, j, k, outside);
                s = s + nbr(x, nx, ny, nz, i + 1, j, k, outside);
                s = s + nbr(x, nx, ny, nz, i, j - 1, k, outside);
                s = s + nbr(x, nx, ny, nz, i, j + 1, k, outside);
                s = s + nbr(x, nx, ny, nz, i, j, k - 1, outside);
                s = s + nbr(x, nx, ny, nz, i, j, k + 1, outside);
                double six = 6.0 * x[IDX(i, j, k)];
                y[IDX(i, j, k)] = s - six;
            }
}

/* Element-sparse 7-point stencil ("element-sparse, where only
 * cells of interest are stored with their connectivity table"; SURVEY.md
 * §8(c) c7): over the active set S,
 *   L_S(x)_i = sum_{j in N6(i)} [j in S ? x_j : outside] - 6 x_i,  i in S;
 * inactive cells of y are set to outside (the host logical view reads
 * inactive cells back as outside). */
void or_sparse_laplace7(int nx, int ny, int nz, const uint8_t *mask, double outside,
                        const double *x, double *y) {
    #pragma omp parallel for schedule(static)
    for (int k = 0; k < nz; ++k)
        for (int j = 0; j < ny; ++j)
            for (int i = 0; i < nx; ++i) {
                int64_t c = IDX(i, j, k);
                if (!mask[c]) {
                    y[c] = outside;
                    continue;
                }
                const int off[6][3] = {{-1, 0, 0}, {1, 0, 0}, {0, -1, 0},
                                       {0, 1, 0},  {0, 0, -1}, {0, 0, 1}};
                double s = 0.0;
                for (int d = 0; d < 6; ++d) {
                    int a = i + off[d][0], b = j + off[d][1], e = k + off[d][2];
                    double v = outside;
                    if (a >= 0 && a < nx && b >= 0 && b < ny && e >= 0 && e < nz && mask[IDX(a, b, e)])
                        v = x[IDX(a, b, e)];
                    s = (d == 0) ? v : s + v;
                }
                double six = 6.0 * x[c];
                y[c] = s - six;
            }
}

/* ---------------------------------------------------------------------- */
/* Config C1 (Fig. 4a; Fig. 1 L33, L43):               */
/*   for k = 1..iters: x <- x + a*y ; y <- L(x) ; d_k = <x, y>             */
/* Dependencies read per L280 (halo on X): map writes X, stencil reads X.  */
/* ---------------------------------------------------------------------- */
void or_c1_loop(int nx, int ny, int nz, double a, int iters, double *x, double *y,
                double *dots) {
    int64_t n = (int64_t)nx * ny * nz;
    for (int k = 0; k < iters; ++k) {
        or_axpy(n, a, y, x);
        or_laplace7(nx, ny, nz, 0.0, x, y);
        dots[k] = or_dot_planes((int64_t)nx * ny, nz, x, y);
    }
}

/* ---------------------------------------------------------------------- */
/* FEM: matrix-free linear-elastic Q1 hexahedra (§VI-C; */
/* SURVEY.md §8(c) c8 readings): unit elements between 2x2x2 node groups,   */
/* 2x2x2 Gauss quadrature, isotropic (E, nu), engineering-strain Voigt     */
/* order (xx, yy, zz, xy, yz, zx).  Local node a = ax + 2ay + 4az,          */
/* dof = 3a + d.                                                           */
/* ---------------------------------------------------------------------- */
void or_fem_ke(double E, double nu, double *Ke /* 24*24 row-major */) {
    double lam = E * nu / ((1.0 + nu) * (1.0 - 2.0 * nu));
    double mu = E / (2.0 * (1.0 + nu));
    double D[6][6];
    memset(D, 0, sizeof(D));
    for (int i = 0; i < 3; ++i)
        for (int j = 0; j < 3; ++j) D[i][j] = lam;
    for (int i = 0; i < 3; ++i) D[i][i] = lam + 2.0 * mu;
    for (int i = 3; i < 6; ++i) D[i][i] = mu;
    memset(Ke, 0, sizeof(double) * 24 * 24);
    double gp[2] = {0.5 - 0.5 / sqrt(3.0), 0.5 + 0.5 / sqrt(3.0)};
    double wgt = 1.0 / 8.0; /* (1/2)^3 on [0,1]^3 */
    for (int gz = 0; gz < 2; ++gz)
        for (int gy = 0; gy < 2; ++gy)
            for (int gx = 0; gx < 2; ++gx) {
                double xi[3] = {gp[gx], gp[gy], gp[gz]};
                double dN[8][3];
                for (int a = 0; a < 8; ++a) {
                    int ax = a & 1, ay = (a >> 1) & 1, az = (a >> 2) & 1;
                    double nxv = ax ? xi[0] : 1.0 - xi[0];
                    double nyv = ay ? xi[1] : 1.0 - xi[1];
                    double nzv = az ? xi[2] : 1.0 - xi[2];
                    double dx = ax ? 1.0 : -1.0, dy = ay ? 1.0 : -1.0, dz = az ? 1.0 : -1.0;
                    dN[a][0] = dx * nyv * nzv;
                    dN[a][1] = nxv * dy * nzv;
                    dN[a][2] = nxv * nyv * dz;
                }
                double B[6][24];
                memset(B, 0, sizeof(B));
                for (int a = 0; a < 8; ++a) {
                    B[0][3 * a + 0] = dN[a][0];
                    B[1][3 * a + 1] = dN[a][1];
                    B[2][3 * a + 2] = dN[a][2];
                    B[3][3 * a + 0] = dN[a][1];
                    B[3][3 * a + 1] = dN[a][0];
                    B[4][3 * a + 1] = dN[a][2];
                    B[4][3 * a + 2] = dN[a][1];
                    B[5][3 * a + 0] = dN[a][2];
                    B[5][3 * a + 2] = dN[a][0];
                }
                double DB[6][24];
                for (int i = 0; i < 6; ++i)
                    for (int c = 0; c < 24; ++c) {
                        double s = 0.0;
                        for (int k = 0; k < 6; ++k) s += D[i][k] * B[k][c];
                        DB[i][c] = s;
                    }
                for (int r = 0; r < 24; ++r)
                    for (int c = 0; c < 24; ++c) {
                        double s = 0.0;
                        for (int k = 0; k < 6; ++k) s += B[k][r] * DB[k][c];
                        Ke[r * 24 + c] += wgt * s;
                    }
            }
}

/* element (ex,ey,ez) exists iff all 8 of its nodes are active (dense: mask NULL) */
static int elem_exists(int nx, int ny, int nz, const uint8_t *mask, int ex, int ey, int ez) {
    if (ex < 0 || ey < 0 || ez < 0 || ex >= nx - 1 || ey >= ny - 1 || ez >= nz - 1) return 0;
    if (!mask) return 1;
    for (int a = 0; a < 8; ++a)
        if (!mask[IDX(ex + (a & 1), ey + ((a >> 1) & 1), ez + ((a >> 2) & 1))]) return 0;
    return 1;
}

/* y = K u with Dirichlet u = 0 on the z = 0 node plane (identity rows and
 * columns: y_D = u_D, free rows ignore Dirichlet columns).  u, y: [3][z][y][x].
 * Element-by-element gather/scatter: y_free += K_e u_e over existing elements.
 * Nodes in no element get y = 0 (plus identity if Dirichlet). */
void or_fem_apply(int nx, int ny, int nz, const double *Ke, const uint8_t *mask,
                  int dirichlet_z0, const double *u, double *y) {
    int64_t n = (int64_t)nx * ny * nz;
    memset(y, 0, sizeof(double) * (size_t)(3 * n));
    /* serial over elements: scatter-add order = element lexicographic order */
    for (int ez = 0; ez < nz - 1; ++ez)
        for (int ey = 0; ey < ny - 1; ++ey)
            for (int ex = 0; ex < nx - 1; ++ex) {
                if (!elem_exists(nx, ny, nz, mask, ex, ey, ez)) continue;
                double ue[24];
                int64_t node[8];
                int fixed[8];
                for (int a = 0; a < 8; ++a) {
                    int i = ex + (a & 1), j = ey + ((a >> 1) & 1), k = ez + ((a >> 2) & 1);
                    node[a] = IDX(i, j, k);
                    fixed[a] = dirichlet_z0 && k == 0;
                    for (int d = 0; d < 3; ++d) ue[3 * a + d] = fixed[a] ? 0.0 : u[node[a] + d * n];
                }
                for (int a = 0; a < 8; ++a) {
                    if (fixed[a]) continue;
                    for (int d = 0; d < 3; ++d) {
                        double s = 0.0;
                        for (int c = 0; c < 24; ++c) s += Ke[(3 * a + d) * 24 + c] * ue[c];
                        y[node[a] + d * n] += s;
                    }
                }
            }
    if (dirichlet_z0)
        for (int j = 0; j < ny; ++j)
            for (int i = 0; i < nx; ++i) {
                int64_t c = IDX(i, j, 0);
                if (mask && !mask[c]) continue;
                for (int d = 0; d < 3; ++d) y[c + d * n] = u[c + d * n];
            }
}

/* Neumann load ("the z = N-1 plane had outward pressure"):
 * uniform pressure p on the +z faces of existing elements that have no
 * existing element above them, as consistent nodal loads for bilinear
 * faces: p*area/4 = p/4 per face node, in +z.  b: [3][z][y][x]. */
void or_fem_rhs(int nx, int ny, int nz, const uint8_t *mask, int dirichlet_z0, double p,
                double *b) {
    int64_t n = (int64_t)nx * ny * nz;
    memset(b, 0, sizeof(double) * (size_t)(3 * n));
    for (int ez = 0; ez < nz - 1; ++ez)
        for (int ey = 0; ey < ny - 1; ++ey)
            for (int ex = 0; ex < nx - 1; ++ex) {
                if (!elem_exists(nx, ny, nz, mask, ex, ey, ez)) continue;
                if (elem_exists(nx, ny, nz, mask, ex, ey, ez + 1)) continue;
                for (int a = 0; a < 4; ++a) {
                    int i = ex + (a & 1), j = ey + ((a >> 1) & 1), k = ez + 1;
                    if (dirichlet_z0 && k == 0) continue;
                    b[IDX(i, j, k) + 2 * n] += 0.25 * p;
                }
            }
}

/* ---------------------------------------------------------------------- */
/* Conjugate gradient (Listing 3 — code lost; textbook  */
/* CG [17] with the UpdateP map moved first, L460):    */
/*   x = x0; r = b - A x0; p = 0; beta = 0; rr = <r,r>; rr0 = rr            */
/*   for k = 1..max_iter:                                                  */
/*     p <- r + beta p ; q <- A p ; pq <- <p,q> (stop if pq <= 0)           */
/*     alpha <- rr/pq ; x <- x + alpha p ; r <- r - alpha q                 */
/*     rr' <- <r,r> ; beta <- rr'/rr ; rr <- rr'                            */
/*     stop if rr == 0 or (rtol > 0 and rr <= rtol^2 rr0)                   */
/* Operators: 0 = Poisson A = -L (7-point, outside 0);                     */
/*            1 = element-sparse A = -L_S (mask);                          */
/*            2 = FEM K (Ke, mask may be NULL, Dirichlet z = 0).            */
/* Vectors live on the full dense logical view ([card][z][y][x]); inactive */
/* cells stay 0 and contribute 0 to every dot.                             */
/* ---------------------------------------------------------------------- */
typedef struct {
    int32_t iters;
    int32_t converged; /* 1 = rtol reached, 2 = rr == 0, 3 = pq <= 0 breakdown */
    double rr0;
    double rr;
} or_cg_result;

static void apply_op(int op, int nx, int ny, int nz, const uint8_t *mask, const double *Ke,
                     const double *p, double *q) {
    int64_t n = (int64_t)nx * ny * nz;
    if (op == 0 || op == 1) {
        if (op == 0)
            or_laplace7(nx, ny, nz, 0.0, p, q);
        else
            or_sparse_laplace7(nx, ny, nz, mask, 0.0, p, q);
        for (int64_t i = 0; i < n; ++i) q[i] = -q[i];
    } else {
        or_fem_apply(nx, ny, nz, Ke, mask, 1, p, q);
    }
}

int or_cg(int op, int nx, int ny, int nz, const uint8_t *mask, const double *Ke,
          const double *b, double *x, int max_iter, double rtol, double *rr_hist,
          or_cg_result *res) {
    int card = (op == 2) ? 3 : 1;
    int64_t n = (int64_t)nx * ny * nz * card;
    int64_t plane = (int64_t)nx * ny;
    int64_t nplanes = (int64_t)nz * card;
    double *r = (double *)malloc(sizeof(double) * (size_t)n);
    double *p = (double *)calloc((size_t)n, sizeof(double));
    double *q = (double *)malloc(sizeof(double) * (size_t)n);
    if (!r || !p || !q) return -1;
    apply_op(op, nx, ny, nz, mask, Ke, x, q);
    for (int64_t i = 0; i < n; ++i) r[i] = b[i] - q[i];
    double beta = 0.0;
    double rr = or_dot_planes(plane, nplanes, r, r);
    double rr0 = rr;
    if (rr_hist) rr_hist[0] = rr;
    res->iters = 0;
    res->converged = (rr == 0.0) ? 2 : 0;
    for (int k = 1; k <= max_iter && !res->converged; ++k) {
        or_axpby(n, 1.0, r, beta, p); /* p <- r + beta p (UpdateP first, L460) */
        apply_op(op, nx, ny, nz, mask, Ke, p, q);
        double pq = or_dot_planes(plane, nplanes, p, q);
        if (!(pq > 0.0)) {
            res->converged = 3;
            break;
        }
        double alpha = rr / pq;
        or_axpy(n, alpha, p, x);
        or_axpy(n, -alpha, q, r);
        double rr_new = or_dot_planes(plane, nplanes, r, r);
        beta = rr_new / rr;
        rr = rr_new;
        res->iters = k;
        if (rr_hist) rr_hist[k] = rr;
        if (rr == 0.0)
            res->converged = 2;
        else if (rtol > 0.0 && rr <= rtol * rtol * rr0)
            res->converged = 1;
    }
    res->rr0 = rr0;
    res->rr = rr;
    free(r);
    free(p);
    free(q);
    return 0;
}

/* ---------------------------------------------------------------------- */
/* D3Q19 BGK, twoPop pull scheme, lid-driven cavity (§VI-A        */
/* L447-L456; formulas absent from the paper — SURVEY.md §8(c) c6):        */
/*  1. gather f_i = fin_i(x - c_i) if inside (or periodic wrap); else       */
/*     half-way bounce-back f_i = fin_opp(i)(x) + [source on lid] 6 w_i     */
/*     rho_w (c_i . u_lid)                                                  */
/*  2. rho = sum f_i ; u = sum c_i f_i / rho                                */
/*  3. feq_i = w_i rho (1 + 3 c.u + 4.5 (c.u)^2 - 1.5 |u|^2)                */
/*  4. fout_i(x) = f_i - omega (f_i - feq_i)                                */
/* The lid is the face y = ny moving in +x; edge/corner sources are        */
/* stationary walls.  bc: 0 = cavity, 1 = periodic.  fin/fout: [19][z][y][x]*/
/* ---------------------------------------------------------------------- */
static const int OR_C[19][3] = {
    {0, 0, 0},  {1, 0, 0},   {-1, 0, 0},  {0, 1, 0},   {0, -1, 0},  {1, 1, 0},  {-1, -1, 0},
    {1, -1, 0}, {-1, 1, 0},  {0, 0, 1},   {1, 0, 1},   {-1, 0, 1},  {0, 1, 1},  {0, -1, 1},
    {0, 0, -1}, {-1, 0, -1}, {1, 0, -1},  {0, -1, -1}, {0, 1, -1}};

void or_lbm_lattice(int *c /* 19*3 */, double *w /* 19 */, int *opp /* 19 */) {
    for (int i = 0; i < 19; ++i) {
        int n2 = 0;
        for (int d = 0; d < 3; ++d) {
            c[3 * i + d] = OR_C[i][d];
            n2 += OR_C[i][d] * OR_C[i][d];
        }
        w[i] = n2 == 0 ? 1.0 / 3.0 : (n2 == 1 ? 1.0 / 18.0 : 1.0 / 36.0);
        for (int j = 0; j < 19; ++j)
            if (OR_C[j][0] == -OR_C[i][0] && OR_C[j][1] == -OR_C[i][1] && OR_C[j][2] == -OR_C[i][2])
                opp[i] = j;
    }
}

/* D3Q19 pull step on an element-sparse domain ("bounce-
 * back where the connectivity table gives -1"): active[z][y][x] != 0 marks
 * fluid cells (NULL: every cell).  A population whose source x - c_i is not an
 * active in-box cell bounces back (half-way, from the opposite population of
 * this cell); the moving-lid term applies only to sources beyond the y = Ny
 * face (the dense reading).  Inactive cells get fout = 0 (they are not
 * stored; the host view reads them back as the outside value 0). */
void or_lbm_step_masked(int nx, int ny, int nz, int bc, double omega, double u_lid, double rho_w,
                        const unsigned char *active, const double *fin, double *fout) {
    int c[57], opp[19];
    double w[19];
    or_lbm_lattice(c, w, opp);
    int64_t n = (int64_t)nx * ny * nz;
    #pragma omp parallel for schedule(static)
    for (int k = 0; k < nz; ++k)
        for (int j = 0; j < ny; ++j)
            for (int i = 0; i < nx; ++i) {
                int64_t cell = IDX(i, j, k);
                double f[19];
                if (active && !active[cell]) {
                    for (int q = 0; q < 19; ++q) fout[(int64_t)q * n + cell] = 0.0;
                    continue;
                }
                for (int q = 0; q < 19; ++q) {
                    int si = i - c[3 * q], sj = j - c[3 * q + 1], sk = k - c[3 * q + 2];
                    if (bc == 1) {
                        si = (si + nx) % nx;
                        sj = (sj + ny) % ny;
                        sk = (sk + nz) % nz;
                        if (active && !active[IDX(si, sj, sk)])
                            f[q] = fin[(int64_t)opp[q] * n + cell];
                        else
                            f[q] = fin[(int64_t)q * n + IDX(si, sj, sk)];
                    } else if (si >= 0 && si < nx && sj >= 0 && sj < ny && sk >= 0 && sk < nz &&
                               (!active || active[IDX(si, sj, sk)])) {
                        f[q] = fin[(int64_t)q * n + IDX(si, sj, sk)];
                    } else {
                        double v = fin[(int64_t)opp[q] * n + cell];
                        int on_lid = (sj == ny) && si >= 0 && si < nx && sk >= 0 && sk < nz;
                        if (on_lid) v = v + 6.0 * w[q] * rho_w * ((double)c[3 * q] * u_lid);
                        f[q] = v;
                    }
                }
                double rho = 0.0, mx = 0.0, my = 0.0, mz = 0.0;
                for (int q = 0; q < 19; ++q) {
                    rho += f[q];
                    mx += c[3 * q] * f[q];
                    my += c[3 * q + 1] * f[q];
                    mz += c[3 * q + 2] * f[q];
                }
                double ux = mx / rho, uy = my / rho, uz = mz / rho;
                double usq = ux * ux + uy * uy + uz * uz;
                for (int q = 0; q < 19; ++q) {
                    double cu = c[3 * q] * ux + c[3 * q + 1] * uy + c[3 * q + 2] * uz;
                    double feq = w[q] * rho * (1.0 + 3.0 * cu + 4.5 * cu * cu - 1.5 * usq);
                    fout[(int64_t)q * n + cell] = f[q] - omega * (f[q] - feq);
                }
            }
}

void or_lbm_step(int nx, int ny, int nz, int bc, double omega, double u_lid, double rho_w,
                 const double *fin, double *fout) {
    or_lbm_step_masked(nx, ny, nz, bc, omega, u_lid, rho_w, 0, fin, fout);
}

/* rho and u (3 components) of a population field f: [19][z][y][x] */
void or_lbm_macroscopic(int nx, int ny, int nz, const double *f, double *rho, double *u) {
    int c[57], opp[19];
    double w[19];
    or_lbm_lattice(c, w, opp);
    int64_t n = (int64_t)nx * ny * nz;
    #pragma omp parallel for schedule(static)
    for (int64_t cell = 0; cell < n; ++cell) {
        double r = 0.0, mx = 0.0, my = 0.0, mz = 0.0;
        for (int q = 0; q < 19; ++q) {
            double v = f[(int64_t)q * n + cell];
            r += v;
            mx += c[3 * q] * v;
            my += c[3 * q + 1] * v;
            mz += c[3 * q + 2] * v;
        }
        rho[cell] = r;
        u[cell] = mx / r;
        u[n + cell] = my / r;
        u[2 * n + cell] = mz / r;
    }
}

/* ---- D2Q9 Karman vortex street (Table I,
 * L398-L439: "2D Karman Vortex Street LBM"; the lattice and boundaries are
 * not stated — readings in DESIGN.md §3):
 *   velocities 0 (0,0); 1 (1,0) 2 (-1,0) 3 (0,1) 4 (0,-1); 5 (1,1) 6 (-1,-1)
 *   7 (1,-1) 8 (-1,1); w = 4/9, 1/9, 1/36; c_s^2 = 1/3.
 *   solid cylinder: (x-cx)^2 + (y-cy)^2 <= r^2 (integers; r < 0: none), half-way
 *   bounce-back; solid cells get fout = 0.
 *   bc 0 (channel): y periodic; a source left of x = 0 gives the inflow
 *   equilibrium f_i^eq(1, (u_in, 0)); a source right of x = nx-1 is clamped
 *   to column nx-1 (zero-gradient outflow).  bc 1: periodic box.
 *   f_i(x) = fin_i(x - c_i) (pull), BGK collide with omega. */
void or_d2q9_lattice(int *c /* 9*2 */, double *w, int *opp) {
    static const int cc[18] = {0, 0, 1, 0, -1, 0, 0, 1, 0, -1, 1, 1, -1, -1, 1, -1, -1, 1};
    static const int oo[9] = {0, 2, 1, 4, 3, 6, 5, 8, 7};
    for (int i = 0; i < 18; ++i) c[i] = cc[i];
    for (int i = 0; i < 9; ++i) {
        opp[i] = oo[i];
        w[i] = i == 0 ? 4.0 / 9.0 : (i < 5 ? 1.0 / 9.0 : 1.0 / 36.0);
    }
}

static double d2q9_feq(const int *c, const double *w, int i, double rho, double ux, double uy) {
    double cu = c[2 * i] * ux + c[2 * i + 1] * uy;
    return w[i] * rho * (1.0 + 3.0 * cu + 4.5 * cu * cu - 1.5 * (ux * ux + uy * uy));
}

void or_d2q9_step(int nx, int ny, int bc, double omega, double u_in, int cx, int cy, int r, const double *fin,
                  double *fout) {
    int c[18], opp[9];
    double w[9];
    or_d2q9_lattice(c, w, opp);
    int64_t n = (int64_t)nx * ny;
    #pragma omp parallel for schedule(static)
    for (int y = 0; y < ny; ++y)
        for (int x = 0; x < nx; ++x) {
            int64_t cell = (int64_t)y * nx + x;
            int64_t dx = x - cx, dy = y - cy;
            if (r >= 0 && dx * dx + dy * dy <= (int64_t)r * r) {
                for (int q = 0; q < 9; ++q) fout[q * n + cell] = 0.0;
                continue;
            }
            double f[9];
            for (int q = 0; q < 9; ++q) {
                int sx = x - c[2 * q], sy = ((y - c[2 * q + 1]) % ny + ny) % ny;
                if (bc == 1) sx = (sx % nx + nx) % nx;
                if (sx < 0) {
                    f[q] = d2q9_feq(c, w, q, 1.0, u_in, 0.0);
                    continue;
                }
                if (sx >= nx) sx = nx - 1;
                int64_t sdx = sx - cx, sdy = sy - cy;
                if (r >= 0 && sdx * sdx + sdy * sdy <= (int64_t)r * r)
                    f[q] = fin[opp[q] * n + cell];
                else
                    f[q] = fin[q * n + (int64_t)sy * nx + sx];
            }
            double rho = 0.0, mx = 0.0, my = 0.0;
            for (int q = 0; q < 9; ++q) {
                rho += f[q];
                mx += c[2 * q] * f[q];
                my += c[2 * q + 1] * f[q];
            }
            double ux = mx / rho, uy = my / rho;
            for (int q = 0; q < 9; ++q) fout[q * n + cell] = f[q] - omega * (f[q] - d2q9_feq(c, w, q, rho, ux, uy));
        }
}
