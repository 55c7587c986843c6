// nb_fem.cu — matrix-free linear-elastic FEM operator and its CG
// (§VI-C: "matrix-free finite-element linear elastic
// solver ... 27 point stencil ... conjugate gradient ... Dirichlet boundary
// conditions fixing displacements to 0 in the z = 0 plane ... the z = N-1
// plane had outward pressure applied").  Readings: SURVEY.md §8(c) c8 /
// Q1 hexahedra of unit size between 2x2x2 node groups,
// 2x2x2 Gauss quadrature, isotropic (E, nu), Dirichlet by identity rows and
// columns, pressure as consistent nodal loads.
//
// Nodes are grid cells; the displacement is a 3-component fp64 SoA field.
//   y_n = sum over existing elements e containing n of K_e u_e (Dirichlet
//         columns dropped), and y_n = u_n on the Dirichlet plane.
// Interior nodes (all 8 elements exist, no Dirichlet neighbour) use the
// assembled 27-block stencil S[o] = sum_{a,b: off(b)-off(a)=o} K_e[a,b]
// (fixed order: o in (dz, dy, dx) lexicographic, then j); surface nodes
// gather element by element (a, then b, then j).  The classification depends
// only on the global node position, so results are partition independent.
#include <cmath>
#include <cstring>

#include "nb_device.cuh"
#include "nb_internal.cuh"

__constant__ double c_ke[24 * 24];      // element stiffness, row-major
__constant__ double c_S[27 * 9];        // interior stencil blocks [o][i][j]

std::vector<std::pair<int, int>> view_ranges(const nb_grid *g, int p, nb_view v);
nb_status nb_halo_exchange_planes(nb_field *f, int c0, int c1, bool send_up, bool send_down, cudaStream_t s);

// K_e of the unit Q1 hexahedron (own implementation; node a = ax + 2 ay + 4 az,
// dof 3a + d, Voigt order xx, yy, zz, xy, yz, zx with engineering shear).
static void fem_element_stiffness(double E, double nu, double *ke) {
    const double lam = E * nu / ((1.0 + nu) * (1.0 - 2.0 * nu)), mu = E / (2.0 * (1.0 + nu));
    double D[6][6] = {};
    for (int i = 0; i < 3; ++i)
        for (int j = 0; j < 3; ++j) D[i][j] = lam + (i == j ? 2.0 * mu : 0.0);
    for (int i = 3; i < 6; ++i) D[i][i] = mu;
    memset(ke, 0, sizeof(double) * 576);
    const double gpt[2] = {0.5 - 0.5 / std::sqrt(3.0), 0.5 + 0.5 / std::sqrt(3.0)};
    for (int q = 0; q < 8; ++q) {
        const double xi = gpt[q & 1], eta = gpt[(q >> 1) & 1], zeta = gpt[(q >> 2) & 1];
        double dN[8][3];
        for (int a = 0; a < 8; ++a) {
            const int ax = a & 1, ay = (a >> 1) & 1, az = (a >> 2) & 1;
            const double fx = ax ? xi : 1 - xi, fy = ay ? eta : 1 - eta, fz = az ? zeta : 1 - zeta;
            dN[a][0] = (ax ? 1.0 : -1.0) * fy * fz;
            dN[a][1] = fx * (ay ? 1.0 : -1.0) * fz;
            dN[a][2] = fx * fy * (az ? 1.0 : -1.0);
        }
        double B[6][24] = {};
        for (int a = 0; a < 8; ++a) {
            B[0][3 * a] = dN[a][0];
            B[1][3 * a + 1] = dN[a][1];
            B[2][3 * a + 2] = dN[a][2];
            B[3][3 * a] = dN[a][1];
            B[3][3 * a + 1] = dN[a][0];
            B[4][3 * a + 1] = dN[a][2];
            B[4][3 * a + 2] = dN[a][1];
            B[5][3 * a] = dN[a][2];
            B[5][3 * a + 2] = dN[a][0];
        }
        for (int r = 0; r < 24; ++r)
            for (int c = 0; c < 24; ++c) {
                double s = 0.0;
                for (int k = 0; k < 6; ++k) {
                    double db = 0.0;
                    for (int l = 0; l < 6; ++l) db += D[k][l] * B[l][c];
                    s += B[k][r] * db;
                }
                ke[r * 24 + c] += s / 8.0;  // weight (1/2)^3
            }
    }
}

static double g_fem_E = -1.0, g_fem_nu = -1.0;

static nb_status fem_upload_constants(double E, double nu) {
    if (E == g_fem_E && nu == g_fem_nu) return NB_OK;
    if (!(E > 0.0) || !(nu > -1.0 && nu < 0.5)) NB_FAIL(NB_EINVAL, "FEM: need E > 0 and -1 < nu < 0.5");
    double ke[576], S[243] = {};
    fem_element_stiffness(E, nu, ke);
    for (int a = 0; a < 8; ++a)
        for (int b = 0; b < 8; ++b) {
            const int ox = (b & 1) - (a & 1), oy = ((b >> 1) & 1) - ((a >> 1) & 1), oz = ((b >> 2) & 1) - ((a >> 2) & 1);
            const int o = (oz + 1) * 9 + (oy + 1) * 3 + (ox + 1);
            for (int i = 0; i < 3; ++i)
                for (int j = 0; j < 3; ++j) S[o * 9 + i * 3 + j] += ke[(3 * a + i) * 24 + 3 * b + j];
        }
    // structural zeros of the assembled stencil: the coupling of components
    // i != j at offset o vanishes unless o_i != 0 and o_j != 0 (odd symmetry
    // of the tensor-product element); store them as exact zeros
    for (int o = 0; o < 27; ++o) {
        const int oc[3] = {o % 3 - 1, (o / 3) % 3 - 1, o / 9 - 1};
        for (int i = 0; i < 3; ++i)
            for (int j = 0; j < 3; ++j)
                if (i != j && (oc[i] == 0 || oc[j] == 0)) S[o * 9 + i * 3 + j] = 0.0;
    }
    NB_CUDA(cudaMemcpyToSymbol(c_ke, ke, sizeof(ke)));
    NB_CUDA(cudaMemcpyToSymbol(c_S, S, sizeof(S)));
    g_fem_E = E;
    g_fem_nu = nu;
    return NB_OK;
}

// K u at node (x, y, zl) of the partition; u: component base pointer and
// stride; returns the 3 components.  Dirichlet nodes (global z = 0) read 0.
__device__ __forceinline__ void fem_node(const double *__restrict__ u, int64_t cs, const PGeo &g, int x, int y, int zl,
                                         double out[3]) {
    const int gz = g.z0 + zl;
    const int64_t c0 = (int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x;
    if (gz == 0) {  // identity row
        out[0] = u[c0];
        out[1] = u[cs + c0];
        out[2] = u[2 * cs + c0];
        return;
    }
    double acc0 = 0.0, acc1 = 0.0, acc2 = 0.0;
    const bool interior = x >= 1 && x <= g.nx - 2 && y >= 1 && y <= g.ny - 2 && gz >= 2 && gz <= g.NZ - 2;
    if (interior) {
#pragma unroll
        for (int o = 0; o < 27; ++o) {
            const int ox = o % 3 - 1, oy = (o / 3) % 3 - 1, oz = o / 9 - 1;
            const int64_t m = c0 + (int64_t)oz * g.ps + (int64_t)oy * g.pitch + ox;
            const double u0 = u[m], u1 = u[cs + m], u2 = u[2 * cs + m];
            const double *S = c_S + o * 9;
            // 153 structurally nonzero coefficients (diagonal blocks always;
            // i-j coupling only where o_i != 0 and o_j != 0): 306 flop/node
            acc0 = fma(S[0], u0, acc0);
            if (ox != 0 && oy != 0) acc0 = fma(S[1], u1, acc0);
            if (ox != 0 && oz != 0) acc0 = fma(S[2], u2, acc0);
            if (oy != 0 && ox != 0) acc1 = fma(S[3], u0, acc1);
            acc1 = fma(S[4], u1, acc1);
            if (oy != 0 && oz != 0) acc1 = fma(S[5], u2, acc1);
            if (oz != 0 && ox != 0) acc2 = fma(S[6], u0, acc2);
            if (oz != 0 && oy != 0) acc2 = fma(S[7], u1, acc2);
            acc2 = fma(S[8], u2, acc2);
        }
    } else {
        for (int a = 0; a < 8; ++a) {
            const int ex = x - (a & 1), ey = y - ((a >> 1) & 1), ez = gz - ((a >> 2) & 1);
            if (ex < 0 || ey < 0 || ez < 0 || ex > g.nx - 2 || ey > g.ny - 2 || ez > g.NZ - 2) continue;
            for (int b = 0; b < 8; ++b) {
                const int mx = ex + (b & 1), my = ey + ((b >> 1) & 1), mz = ez + ((b >> 2) & 1);
                if (mz == 0) continue;  // Dirichlet column
                const int64_t m = (int64_t)(mz - g.z0 + 1) * g.ps + (int64_t)my * g.pitch + mx;
                const double u0 = u[m], u1 = u[cs + m], u2 = u[2 * cs + m];
                const double *K = c_ke + (3 * a) * 24 + 3 * b;
                acc0 = fma(K[0], u0, acc0);
                acc0 = fma(K[1], u1, acc0);
                acc0 = fma(K[2], u2, acc0);
                acc1 = fma(K[24], u0, acc1);
                acc1 = fma(K[25], u1, acc1);
                acc1 = fma(K[26], u2, acc1);
                acc2 = fma(K[48], u0, acc2);
                acc2 = fma(K[49], u1, acc2);
                acc2 = fma(K[50], u2, acc2);
            }
        }
    }
    out[0] = acc0;
    out[1] = acc1;
    out[2] = acc2;
}

// interior fast path needs Dirichlet neighbours excluded: nodes at gz == 1
// have z = 0 neighbours, handled by the surface (element) path above since
// the interior test requires gz >= 2.

enum { FEM_APPLY = 0, FEM_CG_Q = 1, FEM_CG_INIT = 2 };

struct FemArgs {
    const double *u;   // stencil input (x or p)
    const double *b;   // CG init: rhs
    double *y;         // output (y / q / r)
    int64_t cs;
    const CgScal *sc;
};

// one CTA = one 32x8 tile of one plane (canonical dot tiles, per component)
template <int K>
__global__ void __launch_bounds__(DOT_TX *DOT_TY) k_fem(FemArgs A, PGeo g, int zb, double *tp, int T) {
    __shared__ double sw[3][DOT_TY];
    if (K == FEM_CG_Q && A.sc->status != 0) return;
    const int x = blockIdx.x * DOT_TX + threadIdx.x, y = blockIdx.y * DOT_TY + threadIdx.y;
    const int zl = zb + blockIdx.z;
    const bool valid = x < g.nx && y < g.ny;
    double prod[3] = {0.0, 0.0, 0.0};
    if (valid) {
        double o[3];
        fem_node(A.u, A.cs, g, x, y, zl, o);
        const int64_t c0 = (int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x;
#pragma unroll
        for (int c = 0; c < 3; ++c) {
            const int64_t i = c * A.cs + c0;
            if (K == FEM_CG_INIT) {
                const double r = __dsub_rn(A.b[i], o[c]);
                A.y[i] = r;
                prod[c] = __dmul_rn(r, r);
            } else {
                A.y[i] = o[c];
                if (K == FEM_CG_Q) prod[c] = __dmul_rn(A.u[i], o[c]);
            }
        }
    }
    if (K == FEM_APPLY) return;
#pragma unroll
    for (int c = 0; c < 3; ++c) {
        double v = warp_sum_canon(prod[c]);
        if (threadIdx.x == 0) sw[c][threadIdx.y] = v;
    }
    __syncthreads();
    const int t = threadIdx.y * DOT_TX + threadIdx.x;
    if (t < 3) {
        double s = sw[t][0];
#pragma unroll
        for (int w = 1; w < DOT_TY; ++w) s = __dadd_rn(s, sw[t][w]);
        tp[((int64_t)t * g.NZ + g.z0 + zl) * T + blockIdx.y * gridDim.x + blockIdx.x] = s;
    }
}

// CG map: x += alpha_prev p_old (pending), p = r + beta p_old (in place)
__global__ void k_fem_map(double *x, double *p, const double *r, int64_t n, const CgScal *sc) {
    if (sc->status != 0) return;
    const double beta = sc->beta, ap = sc->alpha_prev;
    const int pending = sc->pending;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const double po = p[i];
        if (pending) x[i] = fma(ap, po, x[i]);
        p[i] = fma(beta, po, r[i]);
    }
}

// CG residual update r -= alpha q with per-component canonical tile dots
__global__ void __launch_bounds__(DOT_TX *DOT_TY) k_fem_r(double *r, const double *q, int64_t cs, PGeo g, int zb,
                                                         const CgScal *sc, double *tp, int T) {
    __shared__ double sw[3][DOT_TY];
    if (sc->status != 0) return;
    const double alpha = sc->alpha;
    const int x = blockIdx.x * DOT_TX + threadIdx.x, y = blockIdx.y * DOT_TY + threadIdx.y;
    const int zl = zb + blockIdx.z;
    const bool valid = x < g.nx && y < g.ny;
    const int64_t c0 = (int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x;
#pragma unroll
    for (int c = 0; c < 3; ++c) {
        double prod = 0.0;
        if (valid) {
            const int64_t i = c * cs + c0;
            const double rn = fma(-alpha, q[i], r[i]);
            r[i] = rn;
            prod = __dmul_rn(rn, rn);
        }
        double v = warp_sum_canon(prod);
        if (threadIdx.x == 0) sw[c][threadIdx.y] = v;
    }
    __syncthreads();
    const int t = threadIdx.y * DOT_TX + threadIdx.x;
    if (t < 3) {
        double s = sw[t][0];
#pragma unroll
        for (int w = 1; w < DOT_TY; ++w) s = __dadd_rn(s, sw[t][w]);
        tp[((int64_t)t * g.NZ + g.z0 + zl) * T + blockIdx.y * gridDim.x + blockIdx.x] = s;
    }
}

static inline int64_t fcs(const nb_field *f, int p) { return f->ps * (f->g->parts[p].nz() + 2); }

template <int K>
static nb_status fem_launch(nb_grid *g, int p, FemArgs A, const nb_field *f, int zb, int ze, const char *name) {
    if (ze <= zb) return NB_OK;
    A.cs = fcs(f, p);
    dim3 blk(DOT_TX, DOT_TY), grd(g->tiles_x, g->tiles_y, ze - zb);
    LaunchScope ls(g, g->cs, name);
    k_fem<K><<<grd, blk, 0, g->cs>>>(A, pgeo(f, p), zb, g->tp, g->T);
    return nb_launch_check(name);
}

static nb_status fem_check(const nb_field *u) {
    if (!u) NB_FAIL(NB_EINVAL, "NULL field");
    if (u->g->sparse) NB_FAIL(NB_EUNSUPPORTED, "FEM on element-sparse grids is not built (SURVEY f4)");
    if (u->dt != NB_F64 || u->card != 3) NB_FAIL(NB_EMISMATCH, "FEM fields are fp64 with cardinality 3");
    return NB_OK;
}

extern "C" nb_status nb_fem27_apply(const nb_field *u, nb_field *y, double E, double nu) {
    NB_TRY(fem_check(u));
    NB_TRY(fem_check(y));
    if (u->g != y->g) NB_FAIL(NB_EMISMATCH, "fields belong to different grids");
    nb_grid *g = u->g;
    cudaSetDevice(g->device);
    NB_TRY(fem_upload_constants(E, nu));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        FemArgs A{};
        A.u = (const double *)u->base[p];
        A.y = (double *)y->base[p];
        NB_TRY(fem_launch<FEM_APPLY>(g, p, A, u, 0, g->parts[p].nz(), "k_fem_apply"));
    }
    return NB_OK;
}

// consistent nodal load of pressure p on the top face z = Nz-1 (+z):
// p/4 per adjacent top face, i.e. p * cx * cy / 4 with cx, cy = number of
// adjacent element columns (1 on an edge, 2 inside)
__global__ void k_fem_rhs(double *b, int64_t cs, PGeo g, double pr) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y, zl = blockIdx.z;
    if (x >= g.nx) return;
    const int gz = g.z0 + zl;
    const int64_t c0 = (int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x;
    double v = 0.0;
    if (gz == g.NZ - 1 && gz > 0 && g.nx > 1 && g.ny > 1) {
        const int cx = (x > 0) + (x < g.nx - 1), cy = (y > 0) + (y < g.ny - 1);
        v = pr * (double)(cx * cy) * 0.25;
    }
    b[c0] = 0.0;
    b[cs + c0] = 0.0;
    b[2 * cs + c0] = v;
}

extern "C" nb_status nb_fem27_rhs(nb_field *b, double pressure) {
    NB_TRY(fem_check(b));
    nb_grid *g = b->g;
    cudaSetDevice(g->device);
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        PGeo geo = pgeo(b, p);
        dim3 blk(128), grd((g->nx + 127) / 128, g->ny, geo.nzl);
        LaunchScope ls(g, g->cs, "k_fem_rhs");
        k_fem_rhs<<<grd, blk, 0, g->cs>>>((double *)b->base[p], fcs(b, p), geo, pressure);
        NB_TRY(nb_launch_check("k_fem_rhs"));
    }
    return NB_OK;
}

// ---- CG hooks: map -> halo(p) -> q = K p, <p,q> -> alpha -> r -= alpha q, <r,r> -> beta
nb_status nb_fem_cg_init(nb_cg *cg) {
    nb_grid *g = cg->g;
    NB_TRY(fem_upload_constants(cg->prm.fem_E, cg->prm.fem_nu));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        FemArgs A{};
        A.u = (const double *)cg->x->base[p];
        A.b = (const double *)cg->b->base[p];
        A.y = (double *)cg->r->base[p];
        NB_TRY(fem_launch<FEM_CG_INIT>(g, p, A, cg->x, 0, g->parts[p].nz(), "k_fem_cg_init"));
    }
    return nb_reduce_finalize(g, 3, FIN_CG_INIT, cg->sc, 0);
}

nb_status nb_fem_cg_hooks(nb_cg *cg, int parity) {
    (void)parity;
    nb_grid *g = cg->g;
    nb_field *p_ = cg->p[0];
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        // own planes of all 3 components (halo planes excluded)
        for (int c = 0; c < 3; ++c) {
            int64_t off = (int64_t)c * fcs(p_, p) + p_->ps, n = (int64_t)g->parts[p].nz() * p_->ps;
            LaunchScope ls(g, g->cs, "k_fem_map");
            k_fem_map<<<148 * 8, 256, 0, g->cs>>>((double *)cg->x->base[p] + off, (double *)p_->base[p] + off,
                                                  (const double *)cg->r->base[p] + off, n, cg->sc);
            NB_TRY(nb_launch_check("k_fem_map"));
        }
    }
    NB_TRY(nb_halo_exchange_planes(p_, 0, 3, true, true, g->cs));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        FemArgs A{};
        A.u = (const double *)p_->base[p];
        A.y = (double *)cg->q->base[p];
        A.sc = cg->sc;
        NB_TRY(fem_launch<FEM_CG_Q>(g, p, A, p_, 0, g->parts[p].nz(), "k_fem_cg_q"));
    }
    NB_TRY(nb_reduce_finalize(g, 3, FIN_CG_PQ, cg->sc, 0));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        PGeo geo = pgeo(p_, p);
        dim3 blk(DOT_TX, DOT_TY), grd(g->tiles_x, g->tiles_y, geo.nzl);
        LaunchScope ls(g, g->cs, "k_fem_r");
        k_fem_r<<<grd, blk, 0, g->cs>>>((double *)cg->r->base[p], (const double *)cg->q->base[p], fcs(p_, p), geo, 0,
                                        cg->sc, g->tp, g->T);
        NB_TRY(nb_launch_check("k_fem_r"));
    }
    NB_TRY(nb_reduce_finalize(g, 3, FIN_CG_RR, cg->sc, 0));
    cg->k += 1;
    return NB_OK;
}
