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
#include <cstdlib>
#include <algorithm>
#include <cstring>
#include <type_traits>
#include <vector>

#include "nb_device.cuh"
#include "nb_internal.cuh"
#include "nb_tma.cuh"

__constant__ double c_ke[24 * 24];      // element stiffness, row-major
__constant__ double c_S[27 * 9];        // interior stencil blocks [o][i][j]
__constant__ double c_cv[8];            // its 8 canonical values (see fem_cv_class)

// Structure of the assembled interior stencil (cubic lattice, isotropic
// material): S[o][i][j] = fem_cv_sign * cv[fem_cv_class] for 8 canonical
// values cv, whatever (E, nu).  Diagonal entries depend on the number n of
// nonzero offset components and on whether o_i != 0; off-diagonal entries
// exist only where o_i != 0 and o_j != 0 and carry the sign of o_i o_j.
// fem_upload_constants checks this against the assembled values.
__host__ __device__ constexpr int fem_oc(int o, int i) { return i == 0 ? o % 3 - 1 : i == 1 ? (o / 3) % 3 - 1 : o / 9 - 1; }
__host__ __device__ constexpr int fem_on(int o) { return (fem_oc(o, 0) != 0) + (fem_oc(o, 1) != 0) + (fem_oc(o, 2) != 0); }
__host__ __device__ constexpr int fem_cv_class(int o, int i, int j) {
    return i == j ? (fem_on(o) == 0   ? 0
                     : fem_on(o) == 1 ? (fem_oc(o, i) ? 1 : 2)
                     : fem_on(o) == 2 ? (fem_oc(o, i) ? 3 : 4)
                                      : 5)
                  : (fem_oc(o, i) && fem_oc(o, j)) ? (fem_on(o) == 2 ? 6 : 7) : -1;
}
__host__ __device__ constexpr int fem_cv_sign(int o, int i, int j) { return i == j ? 1 : fem_oc(o, i) * fem_oc(o, j); }
__constant__ const double *c_cls;       // surface-class stencils [FEM_NCLS][27 * 9] (device memory)
// element-sparse node classes: (8-bit mask of the node's existing elements,
// corner a = bit a) * 2 + (gz == 1: Dirichlet columns dropped) [512][27 * 9]
constexpr int FEM_NSCLS = 512;
__constant__ const double *c_scls;
// the surface classes of grids with nx, ny, nz >= 3 (those with all axis
// states in {0, 1, 2} and a non-Dirichlet z state), copied into constant
// memory: a warp whose nodes share a class reads each coefficient with one
// uniform constant-cache load instead of an L1 round trip
constexpr int FEM_NFC = 27;
__constant__ double c_fcls[FEM_NFC][243];

// Surface nodes: y_n = sum over the EXISTING elements around n of K_e u_e
// (an element exists iff its 8 nodes are in the box).  Along one axis, a
// node at coordinate t of N nodes belongs to the elements starting at t - d,
// d in {0, 1}, with 0 <= t - d <= N - 2: the set is {0} at t = 0, {1} at
// t = N - 1, {0, 1} inside and {} when N = 1 — 4 axis states.  Per (x, y, z)
// state and "drop the z = 0 Dirichlet columns" (nodes at gz = 1), the
// assembled 27-block stencil of the existing elements is precomputed once
// (host, fp64), so a surface node costs one 27-point pass instead of the
// 8 x 8 element-pair gather.
constexpr int FEM_NCLS = 4 * 4 * 4 * 2;
__device__ __forceinline__ int fem_axis_state(int t, int n) {
    if (n == 1) return 3;
    return t == 0 ? 0 : (t == n - 1 ? 1 : 2);
}

// constant-memory slot of surface class k = ((xs * 4 + ys) * 4 + zs) * 2 + drop,
// or -1 (degenerate axis, or not a surface class): zs = 2 (drop 0 / 1) or 1
__host__ __device__ __forceinline__ int fem_cslot(int k) {
    const int xs = k >> 5, ys = (k >> 3) & 3, zs = (k >> 1) & 3, d = k & 1;
    if (xs == 3 || ys == 3) return -1;
    const int zk = (zs == 2 && !d) ? 0 : (zs == 1 && !d) ? 1 : (zs == 2 && d) ? 2 : -1;
    if (zk < 0) return -1;
    return zk * 9 + xs * 3 + ys;
}
static int fem_cslot_host(int k) { return fem_cslot(k); }

// coefficient sources of a surface-class stencil
struct FemCConst {
    int slot;
    __device__ __forceinline__ double operator()(int i) const { return c_fcls[slot][i]; }
};
struct FemCGlob {
    const double *__restrict__ p;
    __device__ __forceinline__ double operator()(int i) const { return __ldg(p + i); }
};

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
    // structural zeros of the assembled stencil (the coupling of components
    // i != j at offset o vanishes unless o_i != 0 and o_j != 0) are stored as
    // exact zeros, and every other entry as +-cv[class] (fem_cv_class): the
    // symmetric copies agree to rounding, which is checked here; storing them
    // exactly equal lets the streaming kernel hold 8 values in registers
    double cv[8];
    bool have[8] = {};
    for (int o = 0; o < 27; ++o)
        for (int i = 0; i < 3; ++i)
            for (int j = 0; j < 3; ++j) {
                const int k = fem_cv_class(o, i, j);
                double &e = S[o * 9 + i * 3 + j];
                if (k < 0) {
                    e = 0.0;
                    continue;
                }
                const double v = e * fem_cv_sign(o, i, j);
                if (!have[k]) {
                    cv[k] = v;
                    have[k] = true;
                } else if (std::fabs(v - cv[k]) > 1e-13 * std::fabs(cv[k])) {
                    NB_FAIL(NB_EINVAL, "FEM stencil symmetry check failed (o=%d i=%d j=%d)", o, i, j);
                }
            }
    for (int o = 0; o < 27; ++o)
        for (int i = 0; i < 3; ++i)
            for (int j = 0; j < 3; ++j) {
                const int k = fem_cv_class(o, i, j);
                if (k >= 0) S[o * 9 + i * 3 + j] = fem_cv_sign(o, i, j) > 0 ? cv[k] : -cv[k];
            }
    std::vector<double> cls((size_t)FEM_NCLS * 243, 0.0);
    for (int k = 0; k < FEM_NCLS; ++k) {
        const int drop = k & 1, st[3] = {k >> 5, (k >> 3) & 3, (k >> 1) & 3};  // x, y, z axis states
        auto has = [&](int axis, int d) { return st[axis] == 2 || (st[axis] == 0 && d == 0) || (st[axis] == 1 && d == 1); };
        double *C = cls.data() + (size_t)k * 243;
        for (int a = 0; a < 8; ++a) {  // node n is corner a of the element starting at n - off(a)
            if (!has(0, a & 1) || !has(1, (a >> 1) & 1) || !has(2, (a >> 2) & 1)) continue;
            for (int b = 0; b < 8; ++b) {
                const int ox = (b & 1) - (a & 1), oy = ((b >> 1) & 1) - ((a >> 1) & 1), oz = ((b >> 2) & 1) - ((a >> 2) & 1);
                if (drop && oz == -1) continue;  // Dirichlet column (z = 0)
                const int o = (oz + 1) * 9 + (oy + 1) * 3 + (ox + 1);
                for (int i = 0; i < 3; ++i)
                    for (int j = 0; j < 3; ++j) C[o * 9 + i * 3 + j] += ke[(3 * a + i) * 24 + 3 * b + j];
            }
        }
    }
    // element-sparse classes: the same accumulation (corner a, then b, in
    // increasing order) over the node's existing elements, so a node whose
    // element set is a box surface class gets the very same stencil
    std::vector<double> scls((size_t)FEM_NSCLS * 243, 0.0);
    for (int k = 0; k < FEM_NSCLS; ++k) {
        const int drop = k & 1, em = k >> 1;
        double *C = scls.data() + (size_t)k * 243;
        for (int a = 0; a < 8; ++a) {
            if (!((em >> a) & 1)) continue;
            for (int b = 0; b < 8; ++b) {
                const int ox = (b & 1) - (a & 1), oy = ((b >> 1) & 1) - ((a >> 1) & 1), oz = ((b >> 2) & 1) - ((a >> 2) & 1);
                if (drop && oz == -1) continue;
                const int o = (oz + 1) * 9 + (oy + 1) * 3 + (ox + 1);
                for (int i = 0; i < 3; ++i)
                    for (int j = 0; j < 3; ++j) C[o * 9 + i * 3 + j] += ke[(3 * a + i) * 24 + 3 * b + j];
            }
        }
    }
    static double *d_scls = nullptr;
    if (!d_scls) NB_CUDA(cudaMalloc(&d_scls, sizeof(double) * scls.size()));
    NB_CUDA(cudaMemcpy(d_scls, scls.data(), sizeof(double) * scls.size(), cudaMemcpyHostToDevice));
    NB_CUDA(cudaMemcpyToSymbol(c_scls, &d_scls, sizeof(d_scls)));
    static double *d_cls = nullptr;
    if (!d_cls) NB_CUDA(cudaMalloc(&d_cls, sizeof(double) * cls.size()));
    NB_CUDA(cudaMemcpy(d_cls, cls.data(), sizeof(double) * cls.size(), cudaMemcpyHostToDevice));
    NB_CUDA(cudaMemcpyToSymbol(c_cls, &d_cls, sizeof(d_cls)));
    {
        std::vector<double> fc((size_t)FEM_NFC * 243, 0.0);
        for (int k = 0; k < FEM_NCLS; ++k) {
            const int sl = fem_cslot_host(k);
            if (sl >= 0) std::copy(cls.begin() + (size_t)k * 243, cls.begin() + (size_t)(k + 1) * 243, fc.begin() + (size_t)sl * 243);
        }
        NB_CUDA(cudaMemcpyToSymbol(c_fcls, fc.data(), sizeof(double) * fc.size()));
    }
    NB_CUDA(cudaMemcpyToSymbol(c_ke, ke, sizeof(ke)));
    NB_CUDA(cudaMemcpyToSymbol(c_S, S, sizeof(S)));
    NB_CUDA(cudaMemcpyToSymbol(c_cv, cv, sizeof(cv)));
    g_fem_E = E;
    g_fem_nu = nu;
    return NB_OK;
}

// Operator input accessors: u(c, m, zl) = component c at element offset m,
// which lies in local plane zl.
struct FemUPlain {  // a stored field
    const double *__restrict__ u;
    int64_t cs;
    __device__ __forceinline__ double operator()(int c, int64_t m, int) const { return u[c * cs + m]; }
};
// p_new of the fused CG phase A: fma(beta, p_old, r) inside the slab (the
// arithmetic of k_fem_map), the exchanged p_new on the halo planes
struct FemUCgA {
    const double *__restrict__ r, *__restrict__ po, *__restrict__ pn;
    int64_t cs;
    double beta;
    int nzl;
    __device__ __forceinline__ double operator()(int c, int64_t m, int zl) const {
        const int64_t i = c * cs + m;
        return (zl < 0 || zl >= nzl) ? pn[i] : fma(beta, po[i], r[i]);
    }
};

// surface path of fem_node: the class stencil C over the in-box positions.
// L(ox, oy, oz, u0, u1, u2) fetches the 3 components at offset (ox, oy, oz):
// every caller shares this loop, so the FMA chain (o order, then K + 0..8)
// is the same whichever memory the values come from.
template <class CF, class L>
__device__ __forceinline__ void fem_node_surf_l(const CF &C, const PGeo &g, int x, int y, int gz, const L &load,
                                                double &acc0, double &acc1, double &acc2) {
#pragma unroll
    for (int o = 0; o < 27; ++o) {
        const int ox = o % 3 - 1, oy = (o / 3) % 3 - 1, oz = o / 9 - 1;
        const int mx = x + ox, my = y + oy, mz = gz + oz;
        if (mx < 0 || my < 0 || mz < 0 || mx >= g.nx || my >= g.ny || mz >= g.NZ) continue;
        double u0, u1, u2;
        load(ox, oy, oz, u0, u1, u2);
        const int K = o * 9;
        acc0 = fma(C(K + 0), u0, acc0);
        acc0 = fma(C(K + 1), u1, acc0);
        acc0 = fma(C(K + 2), u2, acc0);
        acc1 = fma(C(K + 3), u0, acc1);
        acc1 = fma(C(K + 4), u1, acc1);
        acc1 = fma(C(K + 5), u2, acc1);
        acc2 = fma(C(K + 6), u0, acc2);
        acc2 = fma(C(K + 7), u1, acc2);
        acc2 = fma(C(K + 8), u2, acc2);
    }
}

template <class CF, class U>
__device__ __forceinline__ void fem_node_surf(const CF &C, const U &u, const PGeo &g, int x, int y, int zl,
                                              double &acc0, double &acc1, double &acc2) {
    const int64_t c0 = (int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x;
    fem_node_surf_l(
        C, g, x, y, g.z0 + zl,
        [&](int ox, int oy, int oz, double &u0, double &u1, double &u2) {
            const int64_t m = c0 + (int64_t)oz * g.ps + (int64_t)oy * g.pitch + ox;
            u0 = u(0, m, zl + oz);
            u1 = u(1, m, zl + oz);
            u2 = u(2, m, zl + oz);
        },
        acc0, acc1, acc2);
}

// surface class of the node at (x, y, gz)
__device__ __forceinline__ int fem_surf_cls(int x, int y, int gz, const PGeo &g) {
    return ((fem_axis_state(x, g.nx) * 4 + fem_axis_state(y, g.ny)) * 4 + fem_axis_state(gz, g.NZ)) * 2 +
           (gz == 1 ? 1 : 0);
}

// K u at node (x, y, zl) of the partition; returns the 3 components.
// Dirichlet nodes (global z = 0) are identity rows.
template <class U>
__device__ __forceinline__ void fem_node(const U &u, const PGeo &g, int x, int y, int zl, double out[3]) {
    const int gz = g.z0 + zl;
    const int64_t c0 = (int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x;
    if (gz == 0) {  // identity row
        out[0] = u(0, c0, zl);
        out[1] = u(1, c0, zl);
        out[2] = u(2, c0, zl);
        return;
    }
    double acc0 = 0.0, acc1 = 0.0, acc2 = 0.0;
    const bool interior = x >= 1 && x <= g.nx - 2 && y >= 1 && y <= g.ny - 2 && gz >= 2 && gz <= g.NZ - 2;
    if (interior) {
#pragma unroll
        for (int o = 0; o < 27; ++o) {
            const int ox = o % 3 - 1, oy = (o / 3) % 3 - 1, oz = o / 9 - 1;
            const int64_t m = c0 + (int64_t)oz * g.ps + (int64_t)oy * g.pitch + ox;
            const double u0 = u(0, m, zl + oz), u1 = u(1, m, zl + oz), u2 = u(2, m, zl + oz);
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
        // surface class stencil (positions outside the box have no element
        // and are skipped; their coefficients are zero)
        const int cls = fem_surf_cls(x, y, gz, g);
        const int sl = fem_cslot(cls);
        if (sl >= 0)
            fem_node_surf(FemCConst{sl}, u, g, x, y, zl, acc0, acc1, acc2);
        else
            fem_node_surf(FemCGlob{c_cls + (size_t)cls * 243}, u, g, x, y, zl, acc0, acc1, acc2);
    }
    out[0] = acc0;
    out[1] = acc1;
    out[2] = acc2;
}

// interior fast path needs Dirichlet neighbours excluded: nodes at gz == 1
// have z = 0 neighbours, handled by the surface (element) path above since
// the interior test requires gz >= 2.

// FEM_CG_A: the fused CG phase A (p_new = r + beta p_old, deferred
// x += alpha_prev p_old, q = K p_new, <p_new, q>) of the TMA schedule
enum { FEM_APPLY = 0, FEM_CG_Q = 1, FEM_CG_INIT = 2, FEM_CG_A = 3 };

struct FemArgs {
    const double *u;   // stencil input (x or p)
    const double *b;   // CG init: rhs
    double *y;         // output (y / q / r)
    int64_t cs;
    const CgScal *sc;
    // FEM_CG_A only: u = p_new is formed on the fly from r and p_old
    const double *r, *po;
    double *pn, *x;
};

template <int K>
__device__ __forceinline__ void fem_node_k(const FemArgs &A, const PGeo &g, int x, int y, int zl, double out[3]) {
    if constexpr (K == FEM_CG_A)
        fem_node(FemUCgA{A.r, A.po, A.pn, A.cs, A.sc->beta, g.nzl}, g, x, y, zl, out);
    else
        fem_node(FemUPlain{A.u, A.cs}, g, x, y, zl, out);
}

// one CTA = one 32x8 tile of one plane (canonical dot tiles, per component)
template <int K>
__global__ void __launch_bounds__(DOT_TX *DOT_TY) k_fem(FemArgs A, PGeo g, int zb, double *tp, int T) {
    __shared__ double sw[3][DOT_TY];
    if ((K == FEM_CG_Q || K == FEM_CG_A) && A.sc->status != 0) return;
    const int x = blockIdx.x * DOT_TX + threadIdx.x, y = blockIdx.y * DOT_TY + threadIdx.y;
    const int zl = zb + blockIdx.z;
    const bool valid = x < g.nx && y < g.ny;
    double prod[3] = {0.0, 0.0, 0.0};
    if (valid) {
        double o[3];
        fem_node(FemUPlain{A.u, A.cs}, g, x, y, zl, o);
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

// ---------------------------------------------------------------------------
// z-marching interior operator (the hot kernel of C5).  A thread owns one
// (x, y) column of a 32x8 tile for ZC planes.  Each u plane is loaded ONCE
// (9 positions x 3 components) and feeds three outputs: plane k-1 (offset
// oz = +1, which completes it), plane k (oz = 0) and plane k+1 (oz = -1,
// which starts it).  Every output therefore receives exactly the FMA chain
// of fem_node's interior path — o = (oz, oy, ox) lexicographic, then j, the
// same structural zeros skipped — so the result is bit-identical to
// fem_node while loading 27 values per node instead of 81 (the L1 / LSU
// pipe, not the FP64 pipe, bounded the one-node-per-thread kernel).
// Nodes outside the interior (column on an x/y face, gz < 2 or gz > NZ-2)
// take fem_node.
// ---------------------------------------------------------------------------
template <int O>
__device__ __forceinline__ void fem_blk(const double (&v)[3], double (&acc)[3]) {
    constexpr int ox = O % 3 - 1, oy = (O / 3) % 3 - 1, oz = O / 9 - 1;
    const double *S = c_S + O * 9;
    acc[0] = fma(S[0], v[0], acc[0]);
    if (ox != 0 && oy != 0) acc[0] = fma(S[1], v[1], acc[0]);
    if (ox != 0 && oz != 0) acc[0] = fma(S[2], v[2], acc[0]);
    if (oy != 0 && ox != 0) acc[1] = fma(S[3], v[0], acc[1]);
    acc[1] = fma(S[4], v[1], acc[1]);
    if (oy != 0 && oz != 0) acc[1] = fma(S[5], v[2], acc[1]);
    if (oz != 0 && ox != 0) acc[2] = fma(S[6], v[0], acc[2]);
    if (oz != 0 && oy != 0) acc[2] = fma(S[7], v[1], acc[2]);
    acc[2] = fma(S[8], v[2], acc[2]);
}

// all 9 in-plane positions of one oz block, in (oy, ox) order
template <int OZ>
__device__ __forceinline__ void fem_plane_blocks(const double (&v)[9][3], double (&acc)[3]) {
    fem_blk<(OZ + 1) * 9 + 0>(v[0], acc);
    fem_blk<(OZ + 1) * 9 + 1>(v[1], acc);
    fem_blk<(OZ + 1) * 9 + 2>(v[2], acc);
    fem_blk<(OZ + 1) * 9 + 3>(v[3], acc);
    fem_blk<(OZ + 1) * 9 + 4>(v[4], acc);
    fem_blk<(OZ + 1) * 9 + 5>(v[5], acc);
    fem_blk<(OZ + 1) * 9 + 6>(v[6], acc);
    fem_blk<(OZ + 1) * 9 + 7>(v[7], acc);
    fem_blk<(OZ + 1) * 9 + 8>(v[8], acc);
}

// load plane k (element offset `base` = centre of the column in that plane)
// and apply it: aA (output k-1) += oz=+1, aB (output k) += oz=0, aC (output
// k+1) = oz=-1 from zero.  cen receives the centre values.
template <bool DA, bool DB>
__device__ __forceinline__ void fem_plane(const double *__restrict__ u, int64_t cs, int64_t base, int64_t pitch,
                                          double (&aA)[3], double (&aB)[3], double (&aC)[3], double (&cen)[3]) {
    double v[9][3];
#pragma unroll
    for (int q = 0; q < 9; ++q) {
        const int64_t m = base + (int64_t)(q / 3 - 1) * pitch + (q % 3 - 1);
        v[q][0] = __ldg(u + m);
        v[q][1] = __ldg(u + cs + m);
        v[q][2] = __ldg(u + 2 * cs + m);
    }
#pragma unroll
    for (int c = 0; c < 3; ++c) cen[c] = v[4][c];
    if (DA) fem_plane_blocks<1>(v, aA);
    if (DB) fem_plane_blocks<0>(v, aB);
    aC[0] = aC[1] = aC[2] = 0.0;
    fem_plane_blocks<-1>(v, aC);
}

template <int K, int ZC>
__global__ void __launch_bounds__(DOT_TX *DOT_TY, 2) k_fem_z(FemArgs A, PGeo g, int zb0, int ze0, double *tp, int T) {
    __shared__ double sw[ZC][3][DOT_TY];
    if ((K == FEM_CG_Q || K == FEM_CG_A) && A.sc->status != 0) return;
    const int x = blockIdx.x * DOT_TX + threadIdx.x, y = blockIdx.y * DOT_TY + threadIdx.y;
    const int zs = zb0 + blockIdx.z * ZC, zend = min(zs + ZC, ze0);
    const bool valid = x < g.nx && y < g.ny;
    const bool colint = x >= 1 && x <= g.nx - 2 && y >= 1 && y <= g.ny - 2;
    // fast planes: interior in z as well (gz in [2, NZ-2])
    int fa = max(zs, 2 - g.z0), fb = min(zend, g.NZ - 1 - g.z0);
    if (!colint || fb < fa) fb = fa;
    const double *__restrict__ u = A.u;
    const int64_t cs = A.cs, col = (int64_t)y * g.pitch + x;
    double aA[3], aB[3], aC[3], cprev[3], ccur[3];
    if (fa < fb) {  // preload planes fa-1 (starts output fa) and fa
        fem_plane<false, false>(u, cs, (int64_t)fa * g.ps + col, g.pitch, aA, aB, aC, cprev);
#pragma unroll
        for (int c = 0; c < 3; ++c) aB[c] = aC[c];
        fem_plane<false, true>(u, cs, (int64_t)(fa + 1) * g.ps + col, g.pitch, aA, aB, aC, ccur);
#pragma unroll
        for (int c = 0; c < 3; ++c) {
            aA[c] = aB[c];
            aB[c] = aC[c];
        }
    }
    for (int zl = zs; zl < zend; ++zl) {
        double o[3] = {0.0, 0.0, 0.0}, uc[3] = {0.0, 0.0, 0.0};
        const int64_t c0 = (int64_t)(zl + 1) * g.ps + col;
        if (zl >= fa && zl < fb) {
            // plane zl+1 completes output zl (held in aA)
            double cnext[3];
            fem_plane<true, true>(u, cs, (int64_t)(zl + 2) * g.ps + col, g.pitch, aA, aB, aC, cnext);
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                o[c] = aA[c];
                uc[c] = ccur[c];
                aA[c] = aB[c];
                aB[c] = aC[c];
                ccur[c] = cnext[c];
            }
        } else if (valid) {
            fem_node(FemUPlain{u, cs}, g, x, y, zl, o);
            if (K == FEM_CG_Q) {
                uc[0] = u[c0];
                uc[1] = u[cs + c0];
                uc[2] = u[2 * cs + c0];
            }
        }
        double prod[3] = {0.0, 0.0, 0.0};
        if (valid) {
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                const int64_t i = c * cs + c0;
                if (K == FEM_CG_INIT) {
                    const double r = __dsub_rn(A.b[i], o[c]);
                    A.y[i] = r;
                    prod[c] = __dmul_rn(r, r);
                } else {
                    A.y[i] = o[c];
                    if (K == FEM_CG_Q) prod[c] = __dmul_rn(uc[c], o[c]);
                }
            }
        }
        if (K != FEM_APPLY) {
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                const double v = warp_sum_canon(prod[c]);
                if (threadIdx.x == 0) sw[zl - zs][c][threadIdx.y] = v;
            }
        }
    }
    (void)cprev;
    if (K == FEM_APPLY) return;
    __syncthreads();
    const int t = threadIdx.y * DOT_TX + threadIdx.x;
    if (t < 3 * (zend - zs)) {
        const int zi = t / 3, c = t % 3;
        double s = sw[zi][c][0];
#pragma unroll
        for (int w = 1; w < DOT_TY; ++w) s = __dadd_rn(s, sw[zi][c][w]);
        tp[((int64_t)c * g.NZ + g.z0 + zs + zi) * T + blockIdx.y * gridDim.x + blockIdx.x] = s;
    }
}

// ---------------------------------------------------------------------------
// TMA-staged z-march (default): the CTA streams its tile's planes (36 x 10
// box per component, tile + ring, fetched by one elected thread with
// cp.async.bulk.tensor into a 4-stage shared-memory ring completed through
// mbarrier transaction bytes) — the per-thread global-load latency that
// stalled k_fem_z disappears; threads read the 27 values of a plane from
// shared memory position by position (3 registers live), so the kernel is
// small enough for 3 CTAs per SM.  Same FMA chains as fem_node (bitwise).
// ---------------------------------------------------------------------------
constexpr int FBX = DOT_TX + 4, FBY = DOT_TY + 2;  // box starts at x0 - 2 (16-byte aligned)
constexpr int FTPAD = 2944;                         // 36*10*8 = 2880 rounded up to 128
constexpr int FNST = 4;
#ifndef NB_FEM_NR
#define NB_FEM_NR 2  // rows per thread of the TMA kernel
#endif
#ifndef NB_FEM_MINB
#define NB_FEM_MINB 5  // CTAs per SM of the TMA kernel (apply / init / q)
#endif
#ifndef NB_FEM_NR_A
#define NB_FEM_NR_A 1  // rows per thread of the fused CG phase A (8 warps per CTA: latency hiding)
#endif
#ifndef NB_FEM_NST_A
#define NB_FEM_NST_A 2  // ring stages of the fused CG phase A (6 component boxes each)
#endif
#ifndef NB_FEM_MINB_A
#define NB_FEM_MINB_A 3
#endif

struct __align__(128) FemStage {
    double c[3][FTPAD / 8];
};

// ---- surface nodes, converged: one thread per node ----------------------
// Surface nodes (an x / y face column, or gz < 2, or gz = NZ-1) are ~2 % of
// the nodes but put one divergent lane into ~17 % of the streaming kernel's
// warps; they are computed first by this kernel (fem_node, raw operator
// output into A.y) and the streaming kernel only reads them back.
struct FemSurf {
    int ncol_edge;  // edge columns of the (x, y) plane
    int nin;        // interior columns (x in [1, nx-2], y in [1, ny-2])
    int nzs;        // z-surface planes of the launch range
    int zlist[3];   // their local plane indices
};

__device__ __forceinline__ void fem_edge_col(int e, int nx, int ny, int &x, int &y) {
    if (e < nx) {
        x = e;
        y = 0;
        return;
    }
    e -= nx;
    if (ny > 1) {
        if (e < nx) {
            x = e;
            y = ny - 1;
            return;
        }
        e -= nx;
    }
    if (nx > 1) {
        y = 1 + e / 2;
        x = (e & 1) ? nx - 1 : 0;
    } else {
        y = 1 + e;
        x = 0;
    }
}

template <int K>
#ifndef NB_FSURF_BX
#define NB_FSURF_BX 128
#endif
__global__ void __launch_bounds__(NB_FSURF_BX) k_fem_surface(FemArgs A, PGeo g, int zb, int ze, FemSurf S,
                                                              int zhi) {
    if ((K == FEM_CG_Q || K == FEM_CG_A) && A.sc->status != 0) return;
    // planes [zb, ze), or with zhi >= 0 the two planes zb and zhi (the
    // boundary planes of a slab in one launch)
    const int nzl = zhi >= 0 ? 2 : ze - zb;
    const int64_t n1 = (int64_t)S.ncol_edge * nzl, n2 = (int64_t)S.nin * S.nzs;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n1 + n2; i += (int64_t)gridDim.x * blockDim.x) {
        int x, y, zl;
        if (i < n1) {  // edge columns: consecutive threads walk along a face (coalesced on y faces)
            fem_edge_col((int)(i % S.ncol_edge), g.nx, g.ny, x, y);
            zl = zb + (int)(i / S.ncol_edge);
            if (zhi >= 0 && zl > zb) zl = zhi;
        } else {
            const int64_t k = i - n1;
            const int c = (int)(k % S.nin);
            zl = S.zlist[k / S.nin];
            x = 1 + c % (g.nx - 2);
            y = 1 + c / (g.nx - 2);
        }
        double o[3];
        fem_node_k<K>(A, g, x, y, zl, o);
        const int64_t c0 = (int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x;
        A.y[c0] = o[0];
        A.y[A.cs + c0] = o[1];
        A.y[2 * A.cs + c0] = o[2];
    }
}

// ---- x-face columns, staged through shared memory ------------------------
// The nodes of the x = 0 and x = nx-1 faces (y in [1, ny-2]) sit one per
// row: a warp of them reads 32 different rows per load, and each value is
// re-read by up to 9 neighbours — k_fem_surface spent most of its time in
// these L1 wavefronts.  Here a CTA of 32 (y) x 8 (z) face nodes first copies
// the 2 x 34 x 10 patch of the 3 components (p_new formed on the fly in CG
// phase A) into shared memory with one load per value, then evaluates the
// same class stencil (fem_node_surf_l: bitwise the global-memory path).
constexpr int XF_Y = 32, XF_Z = 8;

template <int K>
__global__ void __launch_bounds__(XF_Y *XF_Z) k_fem_xface(FemArgs A, PGeo g, int zb, int ze, int zhi) {
    if ((K == FEM_CG_Q || K == FEM_CG_A) && A.sc->status != 0) return;
    if (zhi >= 0) {  // the two planes zb and zhi, one per blockIdx.y
        if (blockIdx.y) zb = zhi;
        ze = zb + 1;
    }
    __shared__ double su[3][XF_Z + 2][XF_Y + 2][2];
    const int face = blockIdx.z;
    const int xa = face ? g.nx - 2 : 0;  // patch columns xa, xa + 1
    const int x = face ? g.nx - 1 : 0;   // node column
    const int ybase = blockIdx.x * XF_Y;  // patch rows ybase .. ybase + 33; nodes ybase + 1 ..
    const int zbase = zhi >= 0 ? zb : zb + blockIdx.y * XF_Z;  // node planes zbase ..; patch planes zbase - 1 ..
    const int tid = threadIdx.x;
    constexpr int NP = (XF_Z + 2) * (XF_Y + 2) * 2;
    for (int e = tid; e < 3 * NP; e += XF_Y * XF_Z) {
        const int c = e / NP, r = e % NP;
        const int xx = r & 1, yy = (r >> 1) % (XF_Y + 2), zz = (r >> 1) / (XF_Y + 2);
        const int yg = ybase + yy, zl = zbase - 1 + zz, gz = g.z0 + zl;
        double v = 0.0;
        if (yg < g.ny && xa + xx < g.nx && gz >= 0 && gz < g.NZ && zl <= g.nzl) {
            const int64_t m = (int64_t)(zl + 1) * g.ps + (int64_t)yg * g.pitch + xa + xx;
            if constexpr (K == FEM_CG_A)
                v = FemUCgA{A.r, A.po, A.pn, A.cs, A.sc->beta, g.nzl}(c, m, zl);
            else
                v = A.u[c * A.cs + m];
        }
        su[c][zz][yy][xx] = v;
    }
    __syncthreads();
    const int ty = tid % XF_Y, tz = tid / XF_Y;
    const int y = ybase + 1 + ty, zl = zbase + tz, gz = g.z0 + zl;
    if (y > g.ny - 2 || zl >= ze) return;
    double o[3];
    if (gz == 0) {  // Dirichlet identity row
#pragma unroll
        for (int c = 0; c < 3; ++c) o[c] = su[c][tz + 1][ty + 1][x - xa];
    } else {
        double a0 = 0.0, a1 = 0.0, a2 = 0.0;
        auto load = [&](int ox, int oy, int oz, double &u0, double &u1, double &u2) {
            const int zz = tz + 1 + oz, yy = ty + 1 + oy, xx = x + ox - xa;
            u0 = su[0][zz][yy][xx];
            u1 = su[1][zz][yy][xx];
            u2 = su[2][zz][yy][xx];
        };
        const int cls = fem_surf_cls(x, y, gz, g);
        const int sl = fem_cslot(cls);
        if (sl >= 0)
            fem_node_surf_l(FemCConst{sl}, g, x, y, gz, load, a0, a1, a2);
        else
            fem_node_surf_l(FemCGlob{c_cls + (size_t)cls * 243}, g, x, y, gz, load, a0, a1, a2);
        o[0] = a0;
        o[1] = a1;
        o[2] = a2;
    }
    const int64_t c0 = (int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x;
    A.y[c0] = o[0];
    A.y[A.cs + c0] = o[1];
    A.y[2 * A.cs + c0] = o[2];
}

// ---- face columns (x or y on the box surface), z-marching -----------------
// One thread per face column and chunk of FZC planes: every u plane is read
// once (its in-box positions of the 3 x 3 neighbourhood) and feeds the three
// outputs it touches, each with its own surface-class stencil; per output
// the in-box positions arrive in o order with all 9 coefficients — the FMA
// chain of fem_node's surface path (bitwise), at ~1/3 of its loads.
constexpr int FZC = 4;

// class code of the output at (x, y, gz): constant slot >= 0, or -1 - class
// (global table)
constexpr int FEM_NOCLS = -1000000;
__device__ __forceinline__ int fem_cls_code(int x, int y, int gz, const PGeo &g) {
    const int cls = ((fem_axis_state(x, g.nx) * 4 + fem_axis_state(y, g.ny)) * 4 + fem_axis_state(gz, g.NZ)) * 2 +
                    (gz == 1 ? 1 : 0);
    const int sl = fem_cslot(cls);
    return sl >= 0 ? sl : -1 - cls;
}

template <class CF>
__device__ __forceinline__ void fem_face_blk(const CF &C, int K, double v0, double v1, double v2, double (&acc)[3]) {
    acc[0] = fma(C(K + 0), v0, acc[0]);
    acc[0] = fma(C(K + 1), v1, acc[0]);
    acc[0] = fma(C(K + 2), v2, acc[0]);
    acc[1] = fma(C(K + 3), v0, acc[1]);
    acc[1] = fma(C(K + 4), v1, acc[1]);
    acc[1] = fma(C(K + 5), v2, acc[1]);
    acc[2] = fma(C(K + 6), v0, acc[2]);
    acc[2] = fma(C(K + 7), v1, acc[2]);
    acc[2] = fma(C(K + 8), v2, acc[2]);
}

__device__ __forceinline__ void fem_face_apply(int code, int K, double v0, double v1, double v2, double (&acc)[3]) {
    if (code >= 0)
        fem_face_blk(FemCConst{code}, K, v0, v1, v2, acc);
    else if (code != FEM_NOCLS)
        fem_face_blk(FemCGlob{c_cls + (size_t)(-1 - code) * 243}, K, v0, v1, v2, acc);
}

// contributions of one plane k (global gz_k) to output accumulators whose
// class codes are CA (output k-1, offset oz = +1), CB (k, 0), CC (k+1, -1)
template <class U>
__device__ __forceinline__ void fem_face_plane(const U &u, const PGeo &g, int x, int y, int k, int CA, int CB, int CC,
                                               double (&aA)[3], double (&aB)[3], double (&aC)[3], double (&cen)[3]) {
    const int64_t base = (int64_t)(k + 1) * g.ps + (int64_t)y * g.pitch + x;
    aC[0] = aC[1] = aC[2] = 0.0;
#pragma unroll
    for (int q = 0; q < 9; ++q) {
        const int oy = q / 3 - 1, ox = q % 3 - 1;
        const int mx = x + ox, my = y + oy;
        if (mx < 0 || my < 0 || mx >= g.nx || my >= g.ny) continue;
        const int64_t m = base + (int64_t)oy * g.pitch + ox;
        const double v0 = u(0, m, k), v1 = u(1, m, k), v2 = u(2, m, k);
        if (q == 4) {
            cen[0] = v0;
            cen[1] = v1;
            cen[2] = v2;
        }
        fem_face_apply(CA, (18 + q) * 9, v0, v1, v2, aA);
        fem_face_apply(CB, (9 + q) * 9, v0, v1, v2, aB);
        fem_face_apply(CC, q * 9, v0, v1, v2, aC);
    }
}

__device__ __forceinline__ void fem_face_col(int c, const PGeo &g, int &x, int &y) {
    const int nyf = g.nx > 2 ? (g.nx - 2) * (g.ny > 1 ? 2 : 1) : 0;  // y-face columns (x interior)
    if (c < nyf) {
        x = 1 + c % (g.nx - 2);
        y = (c / (g.nx - 2)) ? g.ny - 1 : 0;
    } else {
        c -= nyf;
        y = c % g.ny;
        x = (c / g.ny) ? g.nx - 1 : 0;
    }
}

template <class U>
__device__ __forceinline__ void fem_face_col_run(const U &u, const FemArgs &A, const PGeo &g, int x, int y, int zs,
                                                 int zend) {
    double aA[3] = {0.0, 0.0, 0.0}, aB[3] = {0.0, 0.0, 0.0}, aC[3], cen[3], cprev[3] = {0.0, 0.0, 0.0};
    // planes zs-1 .. zend (in-box only: the halo planes beyond the global box are skipped)
    for (int k = zs - 1; k <= zend; ++k) {
        const int gk = g.z0 + k;
        const int oA = k - 1, oB = k, oC = k + 1;  // outputs touched (local planes)
        const bool inA = oA >= zs && oA < zend, inB = oB >= zs && oB < zend, inC = oC >= zs && oC < zend;
        if (gk < 0 || gk >= g.NZ) {  // outside the box: no contribution, just rotate
            aC[0] = aC[1] = aC[2] = 0.0;
            cen[0] = cen[1] = cen[2] = 0.0;
        } else {
            const int CA = inA && g.z0 + oA > 0 ? fem_cls_code(x, y, g.z0 + oA, g) : FEM_NOCLS;
            const int CB = inB && g.z0 + oB > 0 ? fem_cls_code(x, y, g.z0 + oB, g) : FEM_NOCLS;
            const int CC = inC && g.z0 + oC > 0 ? fem_cls_code(x, y, g.z0 + oC, g) : FEM_NOCLS;
            fem_face_plane(u, g, x, y, k, CA, CB, CC, aA, aB, aC, cen);
        }
        if (inA) {  // output k-1 complete
            const int64_t c0 = (int64_t)(oA + 1) * g.ps + (int64_t)y * g.pitch + x;
            const bool ident = g.z0 + oA == 0;  // Dirichlet identity row
#pragma unroll
            for (int cc = 0; cc < 3; ++cc) A.y[cc * A.cs + c0] = ident ? cprev[cc] : aA[cc];
        }
#pragma unroll
        for (int cc = 0; cc < 3; ++cc) {
            aA[cc] = aB[cc];
            aB[cc] = aC[cc];
            cprev[cc] = cen[cc];
        }
    }
}

template <int K>
__global__ void __launch_bounds__(64) k_fem_faces(FemArgs A, PGeo g, int zb, int ze, int ncols) {
    if ((K == FEM_CG_Q || K == FEM_CG_A) && A.sc->status != 0) return;
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= ncols) return;
    int x, y;
    fem_face_col(c, g, x, y);
    const int zs = zb + blockIdx.y * FZC, zend = min(zs + FZC, ze);
    if constexpr (K == FEM_CG_A)
        fem_face_col_run(FemUCgA{A.r, A.po, A.pn, A.cs, A.sc->beta, g.nzl}, A, g, x, y, zs, zend);
    else
        fem_face_col_run(FemUPlain{A.u, A.cs}, A, g, x, y, zs, zend);
}

// ---- streaming interior kernel ---------------------------------------------
// Thread = NR adjacent rows of one x column.  Coefficient-major order: for
// each in-plane position q and each oz block, every coefficient (held in a
// uniform register) is applied to the NR rows back to back, so a constant
// load serves NR nodes.  Per output, positions still arrive in (oy, ox)
// order with the oz blocks in plane order: fem_node's interior FMA chain
// (bitwise).
template <int O, int I, int J, int NR>
__device__ __forceinline__ void fem_cvfma(const double (&cv)[8], const double (&v)[NR][3], double (&acc)[NR][3]) {
    constexpr int k = fem_cv_class(O, I, J);
    if constexpr (k >= 0) {
        // one row per thread (the fused CG phase A): the 8 values sit in
        // registers for the whole kernel; two or more rows (K u, CG set-up):
        // uniform-register operands straight from the constant bank, which
        // measured 1.7 % faster there (0.757 vs 0.770 ms at 384^3) and 2.7 %
        // slower in phase A
        const double c = NR == 1 ? (fem_cv_sign(O, I, J) > 0 ? cv[k] : -cv[k])
                                 : (fem_cv_sign(O, I, J) > 0 ? c_cv[k] : -c_cv[k]);
#pragma unroll
        for (int r = 0; r < NR; ++r) acc[r][I] = fma(c, v[r][J], acc[r][I]);
    }
}

template <int O, int NR>
__device__ __forceinline__ void fem_blkN(const double (&cv)[8], const double (&v)[NR][3], double (&acc)[NR][3]) {
    fem_cvfma<O, 0, 0, NR>(cv, v, acc);
    fem_cvfma<O, 0, 1, NR>(cv, v, acc);
    fem_cvfma<O, 0, 2, NR>(cv, v, acc);
    fem_cvfma<O, 1, 0, NR>(cv, v, acc);
    fem_cvfma<O, 1, 1, NR>(cv, v, acc);
    fem_cvfma<O, 1, 2, NR>(cv, v, acc);
    fem_cvfma<O, 2, 0, NR>(cv, v, acc);
    fem_cvfma<O, 2, 1, NR>(cv, v, acc);
    fem_cvfma<O, 2, 2, NR>(cv, v, acc);
}

// in-plane position Q of the current plane (stage S: 3 component tiles)
// applied to the three outputs it touches: aA (output k-1, oz = +1), aB
// (output k, oz = 0), aC (output k+1, oz = -1); DA / DB: outputs k-1 / k exist
template <int NR, int Q, bool DA, bool DB>
__device__ __forceinline__ void fem_q(const double (&cv)[8], const double *S, int sidx, double (&aA)[NR][3],
                                      double (&aB)[NR][3], double (&aC)[NR][3]) {
    constexpr int off = (Q / 3 - 1) * FBX + (Q % 3 - 1);
    double v[NR][3];
#pragma unroll
    for (int r = 0; r < NR; ++r)
#pragma unroll
        for (int c = 0; c < 3; ++c) v[r][c] = S[c * (FTPAD / 8) + sidx + r * FBX + off];
    if constexpr (DA) fem_blkN<18 + Q, NR>(cv, v, aA);
    if constexpr (DB) fem_blkN<9 + Q, NR>(cv, v, aB);
    fem_blkN<Q, NR>(cv, v, aC);
}

// tensor maps: u = the stencil input (x / p), or r for FEM_CG_A, which also
// streams p_old (po) and, on halo planes, the exchanged p_new (pn)
struct FemMaps {
    CUtensorMap u[3], po[3], pn[3];
};

template <int K>
struct FemTmaCfg {
    static constexpr bool CGA = K == FEM_CG_A;
    static constexpr int NR = CGA ? NB_FEM_NR_A : NB_FEM_NR;  // rows per thread
    static constexpr int NT = DOT_TX * (DOT_TY / NR);         // threads per CTA
    static constexpr int NST = CGA ? NB_FEM_NST_A : FNST;     // ring stages
    static constexpr int SD = (CGA ? 6 : 3) * (FTPAD / 8);    // doubles per stage
    static constexpr int NPB = CGA ? 3 : 0;                    // p_new buffers
    // dynamic shared memory bytes: the ring, plus (FEM_CG_A) the p_new
    // buffers of 3 component tiles each
    static constexpr int SMEM = (NST * SD + NPB * 3 * (FTPAD / 8)) * 8;
    static constexpr int MINB = CGA ? NB_FEM_MINB_A : NB_FEM_MINB;  // CTAs per SM
};

// Which (tile x, tile y, z-chunk) a CTA of the streaming kernel takes.
// mode 0: the whole grid (blockIdx as is); 1: the surface-free box, tiles
// [1, tx-2] x [1, ty-2] of chunks [ca, cb] (grid (tx-2, ty-2, cb-ca+1));
// 2: its complement (1-D grid): every tile of the chunks outside [ca, cb],
// then the ring of edge tiles of each chunk in [ca, cb].
struct FemCtaMap {
    int mode, tx, ty, nc, ca, cb;
};
__device__ __forceinline__ void fem_cta(const FemCtaMap &m, int &bx, int &by, int &ck) {
    if (m.mode == 0) {
        bx = blockIdx.x, by = blockIdx.y, ck = blockIdx.z;
    } else if (m.mode == 1) {
        bx = 1 + blockIdx.x, by = 1 + blockIdx.y, ck = m.ca + blockIdx.z;
    } else {
        int L = blockIdx.x;
        const int tt = m.tx * m.ty, lo = m.ca * tt, hi = (m.nc - 1 - m.cb) * tt;
        if (L < lo || L - lo < hi) {
            ck = L < lo ? L / tt : m.cb + 1 + (L - lo) / tt;
            const int r = (L < lo ? L : L - lo) % tt;
            bx = r % m.tx, by = r / m.tx;
        } else {
            L -= lo + hi;
            const int R = 2 * m.tx + 2 * (m.ty - 2);
            ck = m.ca + L / R;
            int r = L % R;
            if (r < 2 * m.tx) {
                by = r < m.tx ? 0 : m.ty - 1, bx = r % m.tx;
            } else {
                r -= 2 * m.tx;
                bx = (r & 1) ? m.tx - 1 : 0, by = 1 + (r >> 1);
            }
        }
    }
}

// Per-CTA state of the streaming kernel.  A thread owns NR rows of one x
// column of a 32 x 8 tile and marches ZC output planes; plane j of the
// chunk (local plane zs - 1 + j) arrives in ring stage j % NST.
template <int K, int ZC>
struct FemTma {
    using Cfg = FemTmaCfg<K>;
    static constexpr bool CGA = Cfg::CGA;
    static constexpr int NR = Cfg::NR, NT = Cfg::NT, NST = Cfg::NST, SD = Cfg::SD, CP = FTPAD / 8;
    const FemMaps &M;
    const FemArgs &A;
    const PGeo &g;
    double *fsm;
    uint64_t *bar;
    double (*sw)[3][DOT_TY];  // [output parity][component][tile row]
    double *tp;
    int T;
    int tid, lane, x0, y0, x, ya, zs, zend, nplanes, fa, fb, sidx, bx, by, tx;
    bool xin, xint, anyfast, dox, ctaint;
    int64_t cb;  // (ya, x) offset within a plane
    double beta, ap;
    double cv[8];  // canonical stencil values (registers for the whole kernel)

    __device__ __forceinline__ bool halo(int zl) const { return zl < 0 || zl >= g.nzl; }

    __device__ __forceinline__ void issue(int j) const {  // plane zs-1+j -> stage j % NST
        double *S = fsm + ((unsigned)j % NST) * SD;
        uint64_t *b = &bar[(unsigned)j % NST];
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        const int zl = zs - 1 + j, tz = zl + 1;
        if (CGA && !halo(zl)) {
            mbar_expect_tx(b, 6 * FBX * FBY * 8);
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                tma_load_3d(S + c * CP, &M.u[c], b, x0 - 2, y0 - 1, tz);
                tma_load_3d(S + (3 + c) * CP, &M.po[c], b, x0 - 2, y0 - 1, tz);
            }
        } else {
            mbar_expect_tx(b, 3 * FBX * FBY * 8);
#pragma unroll
            for (int c = 0; c < 3; ++c) tma_load_3d(S + c * CP, CGA ? &M.pn[c] : &M.u[c], b, x0 - 2, y0 - 1, tz);
        }
    }

    // plane j: its contributions to outputs j-2 (aA), j-1 (aB), j (aC, fresh);
    // output j-2 is then complete (centre values cP, of plane j-1); cC
    // receives this plane's centre values.
    // FEM_CG_A: the raw stage (r, p_old) is first turned into p_new in one of
    // two p_new buffers (double-buffered: one barrier per plane), so the
    // stage is refilled while the FMAs run; the deferred x update is applied
    // after the FMAs, which hide the latency of the x loads.
    template <bool DA, bool DB>
    __device__ __forceinline__ void step(int j, double (&aA)[NR][3], double (&aB)[NR][3], double (&aC)[NR][3],
                                         const double (&cP)[NR][3], double (&cC)[NR][3]) const {
        const int zin = zs - 1 + j;  // local plane held by this stage
        const bool own = zin >= zs && zin < zend;
        const double *S = fsm + ((unsigned)j % NST) * SD;  // stencil input tiles of this plane
        double xo[NR][3], pc[NR][3];               // CGA: x and p_old of the own centres
        if constexpr (CGA) {
            if (own && dox) {
                const double *xp = A.x + (int64_t)(zin + 1) * g.ps + cb;
#pragma unroll
                for (int r = 0; r < NR; ++r) {
                    const bool v = ctaint || (xin && ya + r < g.ny);
#pragma unroll
                    for (int c = 0; c < 3; ++c) xo[r][c] = v ? __ldcs(xp + c * A.cs + r * g.pitch) : 0.0;
                }
            }
            mbar_wait(&bar[(unsigned)j % NST], ((unsigned)j / NST) & 1u);
            // p_new tiles, three buffers: plane j's is formed here; plane j-1's
            // stays readable for this step's epilogue (its centres are the dot's
            // p_new), and is overwritten only at step j+2, past barrier j+1
            double *P = fsm + NST * SD + ((unsigned)j % 3u) * 3 * CP;
            // the three component boxes are contiguous (r at S, p_old at
            // S + 3 CP, p_new at P): one flat 16-byte pass over 3 CP doubles
            // (the 8 padding doubles of a box are never read)
            constexpr int NP2 = 3 * CP / 2, NIT = (NP2 + NT - 1) / NT;
            const double2 *S2 = reinterpret_cast<const double2 *>(S);
            double2 *P2 = reinterpret_cast<double2 *>(P);
            if (!halo(zin)) {  // CTA-uniform
#pragma unroll
                for (int k = 0; k < NIT; ++k) {
                    const int e = tid + k * NT;
                    if (NP2 % NT == 0 || k + 1 < NIT || e < NP2) {
                        const double2 rv = S2[e], pv = S2[NP2 + e];
                        P2[e] = make_double2(fma(beta, pv.x, rv.x), fma(beta, pv.y, rv.y));
                    }
                }
#pragma unroll
                for (int r = 0; r < NR; ++r)
#pragma unroll
                    for (int c = 0; c < 3; ++c) pc[r][c] = S[(3 + c) * CP + sidx + r * FBX];
            } else {
#pragma unroll
                for (int k = 0; k < NIT; ++k) {
                    const int e = tid + k * NT;
                    if (NP2 % NT == 0 || k + 1 < NIT || e < NP2) P2[e] = S2[e];
                }
            }
            __syncthreads();  // p_new tiles ready; the raw stage is free; step j-1's dot rows are in sw
            if (tid == 0 && j + NST < nplanes) issue(j + NST);
            if (j >= 3) flush(zs + j - 3, tp, T);
            S = P;
        } else {
            if (j >= 3) flush(zs + j - 3, tp, T);  // the previous step's output (barrier passed)
            mbar_wait(&bar[(unsigned)j % NST], ((unsigned)j / NST) & 1u);
        }
        if (anyfast) {
#pragma unroll
            for (int r = 0; r < NR; ++r) aC[r][0] = aC[r][1] = aC[r][2] = 0.0;
            fem_q<NR, 0, DA, DB>(cv, S, sidx, aA, aB, aC);
            fem_q<NR, 1, DA, DB>(cv, S, sidx, aA, aB, aC);
            fem_q<NR, 2, DA, DB>(cv, S, sidx, aA, aB, aC);
            fem_q<NR, 3, DA, DB>(cv, S, sidx, aA, aB, aC);
            fem_q<NR, 4, DA, DB>(cv, S, sidx, aA, aB, aC);
            fem_q<NR, 5, DA, DB>(cv, S, sidx, aA, aB, aC);
            fem_q<NR, 6, DA, DB>(cv, S, sidx, aA, aB, aC);
            fem_q<NR, 7, DA, DB>(cv, S, sidx, aA, aB, aC);
            fem_q<NR, 8, DA, DB>(cv, S, sidx, aA, aB, aC);
        }
        if constexpr (!CGA) {
#pragma unroll
            for (int r = 0; r < NR; ++r)
#pragma unroll
                for (int c = 0; c < 3; ++c) cC[r][c] = S[c * CP + sidx + r * FBX];
        }
        if constexpr (CGA) {
            if (own) {  // own plane: store p_new and the deferred x += alpha_prev p_old
                const int64_t c0 = (int64_t)(zin + 1) * g.ps + cb;
#pragma unroll
                for (int r = 0; r < NR; ++r) {
                    if (ctaint || (xin && ya + r < g.ny)) {
                        const int64_t cr = c0 + r * g.pitch;
#pragma unroll
                        for (int c = 0; c < 3; ++c) {
                            __stcs(A.pn + c * A.cs + cr, S[c * CP + sidx + r * FBX]);  // S = this plane's p_new tiles
                            if (dox) __stcs(A.x + c * A.cs + cr, fma(ap, pc[r][c], xo[r][c]));
                        }
                    }
                }
            }
        }
        if constexpr (DA) {
            if constexpr (CGA) {  // centres of output j-2 = plane j-1, read back from its p_new buffer
                const double *Pp = fsm + NST * SD + ((unsigned)(j + 2) % 3u) * 3 * CP;
                double cen[NR][3];
#pragma unroll
                for (int r = 0; r < NR; ++r)
#pragma unroll
                    for (int c = 0; c < 3; ++c) cen[r][c] = Pp[c * CP + sidx + r * FBX];
                epilogue(j - 2 + zs, aA, cen);
            } else {
                epilogue(j - 2 + zs, aA, cP);
            }
        }
        if constexpr (!CGA) {
            __syncthreads();  // stage j % NST is free
            if (tid == 0 && j + NST < nplanes) issue(j + NST);
        }
    }

    // tile partials of output zl (its 8 row sums, after a barrier): rows in
    // increasing y; sw is double-buffered by output parity
    __device__ __forceinline__ void flush(int zl, double *tp, int T) const {
        if (K != FEM_APPLY && tid < 3) {
            const double(*w)[DOT_TY] = sw[(zl - zs) & 1];
            double s = w[tid][0];
#pragma unroll
            for (int k = 1; k < DOT_TY; ++k) s = __dadd_rn(s, w[tid][k]);
            tp[((int64_t)tid * g.NZ + g.z0 + zl) * T + by * tx + bx] = s;
        }
    }

    // output plane zl: store (or, for surface nodes, read back), dot partials
    __device__ __forceinline__ void epilogue(int zl, const double (&o3)[NR][3], const double (&cen)[NR][3]) const {
        const bool zfast = zl >= fa && zl < fb;
        double prod[NR * 3];
        if (K != FEM_CG_INIT && ctaint && zfast) {  // CTA-uniform: every node of the tile is interior
            const int64_t c0 = (int64_t)(zl + 1) * g.ps + cb;
#pragma unroll
            for (int r = 0; r < NR; ++r)
#pragma unroll
                for (int c = 0; c < 3; ++c) {
                    __stcs(A.y + c * A.cs + c0 + r * g.pitch, o3[r][c]);
                    prod[r * 3 + c] = (K == FEM_CG_Q || CGA) ? __dmul_rn(cen[r][c], o3[r][c]) : 0.0;
                }
        } else
#pragma unroll
        for (int r = 0; r < NR; ++r) {
            const int y = ya + r;
            const bool valid = xin && y < g.ny;
            const bool fast = zfast && xint && y >= 1 && y <= g.ny - 2;
            const int64_t c0 = (int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x;
            double o[3] = {o3[r][0], o3[r][1], o3[r][2]};
            if (valid && !fast)  // computed by k_fem_surface / k_fem_faces
#pragma unroll
                for (int c = 0; c < 3; ++c) o[c] = A.y[c * A.cs + c0];
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                double pr = 0.0;
                if (valid) {
                    const int64_t i = c * A.cs + c0;
                    if (K == FEM_CG_INIT) {
                        const double rr = __dsub_rn(A.b[i], o[c]);
                        A.y[i] = rr;
                        pr = __dmul_rn(rr, rr);
                    } else {
                        if (fast) __stcs(A.y + i, o[c]);
                        if (K == FEM_CG_Q || CGA) pr = __dmul_rn(cen[r][c], o[c]);
                    }
                }
                prod[r * 3 + c] = pr;
            }
        }
        if (K != FEM_APPLY) {
            constexpr int NV = NR * 3, M2 = WarpMulti<NV>::M;
            const double v = warp_sum_multi<NV>(prod, lane);
            const int i = warp_multi_index<NV>(lane);
            if (i < NV && (lane & (32 / M2 - 1)) == 0) sw[(zl - zs) & 1][i % 3][threadIdx.y * NR + i / 3] = v;
        }
    }
};

template <int K, int ZC, int NR>
__global__ void __launch_bounds__(FemTmaCfg<K>::NT, FemTmaCfg<K>::MINB)
    k_fem_tma(const __grid_constant__ FemMaps M, FemArgs A, PGeo g, int zb0, int ze0, double *tp, int T, FemCtaMap cm) {
    using Cfg = FemTmaCfg<K>;
    static_assert(Cfg::NR == NR, "rows per thread");
    extern __shared__ __align__(128) double fsm[];
    __shared__ __align__(8) uint64_t bar[Cfg::NST];
    __shared__ double sw[2][3][DOT_TY];
    if ((K == FEM_CG_Q || K == FEM_CG_A) && A.sc->status != 0) return;
    FemTma<K, ZC> t{M, A, g, fsm, bar, sw, tp, T};
    t.tid = threadIdx.y * DOT_TX + threadIdx.x;
    t.lane = threadIdx.x;
    {
        int ck;
        fem_cta(cm, t.bx, t.by, ck);
        t.tx = cm.tx;
        t.zs = zb0 + ck * ZC;
    }
    t.x0 = t.bx * DOT_TX;
    t.y0 = t.by * DOT_TY;
    t.x = t.x0 + threadIdx.x;
    t.ya = t.y0 + threadIdx.y * NR;  // rows ya .. ya+NR-1
    t.zend = min(t.zs + ZC, ze0);
    t.nplanes = t.zend - t.zs + 2;  // planes zs-1 .. zend
    t.xin = t.x < g.nx;
    t.xint = t.x >= 1 && t.x <= g.nx - 2;
    t.fa = max(t.zs, 2 - g.z0);  // fast outputs [fa, fb)
    t.fb = min(t.zend, g.NZ - 1 - g.z0);
    t.anyfast = false;
#pragma unroll
    for (int r = 0; r < NR; ++r) t.anyfast |= t.xint && t.ya + r >= 1 && t.ya + r <= g.ny - 2;
    // the whole 32 x 8 tile is x/y-interior (no surface node, no row past ny)
    t.ctaint = t.x0 >= 1 && t.x0 + DOT_TX <= g.nx - 1 && t.y0 >= 1 && t.y0 + DOT_TY <= g.ny - 1;
    t.cb = (int64_t)t.ya * g.pitch + t.x;
    t.sidx = (threadIdx.y * NR + 1) * FBX + threadIdx.x + 2;
    t.beta = t.ap = 0.0;
    t.dox = false;
#pragma unroll
    for (int k = 0; k < 8; ++k) t.cv[k] = NR == 1 ? c_cv[k] : 0.0;
    if constexpr (K == FEM_CG_A) {
        t.beta = A.sc->beta;
        t.ap = A.sc->alpha_prev;
        t.dox = A.sc->pending != 0;
    }
    if (t.tid == 0) {
        for (int k = 0; k < Cfg::NST; ++k) mbar_init(&bar[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (t.tid == 0)
        for (int j = 0; j < min(Cfg::NST, t.nplanes); ++j) t.issue(j);
    // accumulators and centre values rotate through three register sets:
    // the plane loop is unrolled by three so the rotation is free
    double a0[NR][3], a1[NR][3], a2[NR][3], c0[NR][3], c1[NR][3], c2[NR][3];
#pragma unroll
    for (int r = 0; r < NR; ++r)
#pragma unroll
        for (int c = 0; c < 3; ++c) a0[r][c] = a1[r][c] = a2[r][c] = c0[r][c] = c1[r][c] = c2[r][c] = 0.0;
    // plane 0 starts output 0 (a1 after rotation), plane 1 ...
    t.template step<false, false>(0, a2, a0, a1, c2, c0);
    t.template step<false, true>(1, a0, a1, a2, c0, c1);
    int j = 2;
#pragma unroll 1
    for (; j + 2 < t.nplanes; j += 3) {
        t.template step<true, true>(j, a1, a2, a0, c1, c2);
        t.template step<true, true>(j + 1, a2, a0, a1, c2, c0);
        t.template step<true, true>(j + 2, a0, a1, a2, c0, c1);
    }
    if (j < t.nplanes) t.template step<true, true>(j, a1, a2, a0, c1, c2);
    if (j + 1 < t.nplanes) t.template step<true, true>(j + 1, a2, a0, a1, c2, c0);
    if constexpr (K == FEM_CG_A) __syncthreads();
    t.flush(t.zend - 1, tp, T);  // the last output (after a barrier)
}

// CG map: x += alpha_prev p_old (pending, when dox), p_new = r + beta p_old,
// over `nseg` runs of n elements starting at off[blockIdx.y] (all boundary
// planes x components of a partition in one launch)
struct FemMapSegs {
    int64_t off[8];
};
__global__ void k_fem_map(double *x, double *pn, const double *po, const double *r, FemMapSegs S, int64_t n,
                          const CgScal *sc, int dox) {
    if (sc->status != 0) return;
    const double beta = sc->beta, ap = sc->alpha_prev;
    const int pending = dox && sc->pending;
    const int64_t o = S.off[blockIdx.y];
    x += o, pn += o, po += o, r += o;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const double pv = po[i];
        if (pending) x[i] = fma(ap, pv, x[i]);
        pn[i] = fma(beta, pv, r[i]);
    }
}

// CG residual update, z-marching: a CTA owns one 32 x 8 tile for FRZ planes;
// the next plane's q and r are loaded while the current one is updated, and
// the three component dots of a plane go through one transposed butterfly
// (bitwise the three canonical butterflies of k_fem_r)
constexpr int FRZ = 16;
__global__ void __launch_bounds__(DOT_TX *DOT_TY) k_fem_rz(double *r, const double *q, int64_t cs, PGeo g, int zb, int ze,
                                                          const CgScal *sc, double *tp, int T) {
    __shared__ double sw[FRZ][3][DOT_TY];
    if (sc->status != 0) return;
    const double alpha = sc->alpha;
    const int lane = threadIdx.x, w = threadIdx.y;
    const int x = blockIdx.x * DOT_TX + lane, y = blockIdx.y * DOT_TY + w;
    const int zs = zb + blockIdx.z * FRZ, zend = min(ze, zs + FRZ);
    const bool valid = x < g.nx && y < g.ny;
    const int64_t ps = g.ps, off = (int64_t)(zs + 1) * ps + (int64_t)y * g.pitch + x;
    const double *qp = q + off;
    double *rp = r + off;
    double qn[3] = {0.0, 0.0, 0.0}, rn[3] = {0.0, 0.0, 0.0};
    if (valid)
#pragma unroll
        for (int c = 0; c < 3; ++c) {
            qn[c] = __ldcs(qp + c * cs);
            rn[c] = __ldcs(rp + c * cs);
        }
    for (int z = zs; z < zend; ++z) {
        double qc[3], rc[3];
#pragma unroll
        for (int c = 0; c < 3; ++c) qc[c] = qn[c], rc[c] = rn[c];
        if (valid && z + 1 < zend)
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                qn[c] = __ldcs(qp + ps + c * cs);
                rn[c] = __ldcs(rp + ps + c * cs);
            }
        double prod[3] = {0.0, 0.0, 0.0};
        if (valid)
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                const double v = fma(-alpha, qc[c], rc[c]);
                __stcs(rp + c * cs, v);
                prod[c] = __dmul_rn(v, v);
            }
        const double s = warp_sum_multi<3>(prod, lane);
        const int i = warp_multi_index<3>(lane);
        if ((lane & 7) == 0 && i < 3) sw[z - zs][i][w] = s;
        qp += ps;
        rp += ps;
    }
    __syncthreads();
    const int t = w * DOT_TX + lane;
    if (t < 3 * (zend - zs)) {
        const int zi = t / 3, c = t % 3;
        double s = sw[zi][c][0];
#pragma unroll
        for (int k = 1; k < DOT_TY; ++k) s = __dadd_rn(s, sw[zi][c][k]);
        tp[((int64_t)c * g.NZ + g.z0 + zs + zi) * T + blockIdx.y * gridDim.x + blockIdx.x] = s;
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

static inline int64_t fcs(const nb_field *f, int p) { return nb_cstride(f, p); }

// what: FEM_SURF = only the surface-node kernels of the TMA path, FEM_BULK =
// only the streaming kernel, FEM_ALL = both (the OCC schedule runs the
// surface nodes of the interior planes while the halo is in flight)
enum { FEM_SURF = 1, FEM_BULK = 2, FEM_ALL = 3 };

#ifndef NB_FEM_ZC
#define NB_FEM_ZC 32  // planes per CTA of the TMA z-march
#endif
template <int K>
static nb_status fem_launch(nb_grid *g, int p, FemArgs A, const nb_field *f, int zb, int ze, const char *name,
                            int what = FEM_ALL, int zhi = -1) {
    if (ze <= zb) return NB_OK;
    if (zhi >= 0 && (what != FEM_SURF || ze != zb + 1 || zhi <= zb)) NB_FAIL(NB_EINVAL, "fem_launch: bad plane pair");
    A.cs = fcs(f, p);
    const PGeo geo = pgeo(f, p);
    const char *variant = getenv("NB_FEM_KERNEL");  // "plain" | "zmarch" | default TMA
    if (variant && !strcmp(variant, "plain")) {  // the one-node-per-thread reference kernel
        dim3 blk(DOT_TX, DOT_TY), grd(g->tiles_x, g->tiles_y, ze - zb);
        LaunchScope ls(g, g->cs, name);
        k_fem<K><<<grd, blk, 0, g->cs>>>(A, geo, zb, g->tp, g->T);
    } else if (!variant && nb_tma_enabled()) {
        using Cfg = FemTmaCfg<K>;
        constexpr int ZC = NB_FEM_ZC, NR = Cfg::NR;
        FemMaps M;
        if constexpr (K == FEM_CG_A) {
            for (int c = 0; c < 3; ++c) {
                NB_TRY(tmap_for(A.r + c * A.cs, geo, 0, &M.u[c]));
                NB_TRY(tmap_for(A.po + c * A.cs, geo, 0, &M.po[c]));
                NB_TRY(tmap_for(A.pn + c * A.cs, geo, 0, &M.pn[c]));
            }
        } else {
            for (int c = 0; c < 3; ++c) NB_TRY(tmap_for(A.u + c * A.cs, geo, 0, &M.u[c]));
        }
        // surface nodes first (converged), then the streaming interior.
        // NB_FEM_CONC (default on): the surface kernels run on the halo
        // stream concurrently with the streaming kernel's surface-free box
        // (interior tiles of the chunks without a z-surface plane: its
        // epilogue never reads a surface node's output); the rest of the
        // streaming kernel waits for them on a side stream, and the grid
        // stream joins both.  Same CTAs, same arithmetic: same bits.
        const int tx = g->tiles_x, ty = g->tiles_y, nck = (ze - zb + ZC - 1) / ZC;
        FemCtaMap cm{0, tx, ty, nck, 0, -1};
        bool conc = false;
        {
            const char *cv = getenv("NB_FEM_CONC");
            if ((!cv || atoi(cv) != 0) && (what == FEM_ALL) && zhi < 0 && tx >= 3 && ty >= 3) {
                // chunks free of z-surface planes (global z < 2 or z > NZ-2)
                int ca = 0, cb = nck - 1;
                while (ca < nck && (geo.z0 + zb + ca * ZC < 2 || geo.z0 + std::min(zb + (ca + 1) * ZC, ze) - 1 > geo.NZ - 2)) ++ca;
                while (cb >= ca && (geo.z0 + zb + cb * ZC < 2 || geo.z0 + std::min(zb + (cb + 1) * ZC, ze) - 1 > geo.NZ - 2)) --cb;
                if (cb >= ca) {
                    cm.ca = ca, cm.cb = cb;
                    conc = true;
                }
            }
        }
        cudaStream_t ss = g->cs;  // stream of the surface kernels
        if (conc) {
            if (!g->fs) {
                int lo, hi;
                NB_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
                NB_CUDA(cudaStreamCreateWithPriority(&g->fs, cudaStreamNonBlocking, hi));
                for (auto &e : g->fev) NB_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
            }
            NB_CUDA(cudaEventRecord(g->fev[0], g->cs));  // fork
            NB_CUDA(cudaStreamWaitEvent(g->hs, g->fev[0], 0));
            NB_CUDA(cudaStreamWaitEvent(g->fs, g->fev[0], 0));
            ss = g->hs;
        }
        cudaStream_t xs = conc ? g->fs : ss;  // x-face kernel: its own stream (starts with k_fem_surface)
        FemSurf S{};
        const int nx = geo.nx, ny = geo.ny;
        S.ncol_edge = nx * std::min(ny, 2) + std::max(ny - 2, 0) * std::min(nx, 2);
        S.nin = std::max(nx - 2, 0) * std::max(ny - 2, 0);
        for (int zl = zb; zl < ze; ++zl) {
            const int gz = geo.z0 + zl;
            if (gz < 2 || gz > geo.NZ - 2) S.zlist[S.nzs++] = zl;
        }
        if (zhi >= 0 && (geo.z0 + zhi < 2 || geo.z0 + zhi > geo.NZ - 2)) S.zlist[S.nzs++] = zhi;
        const int nzr = zhi >= 0 ? 2 : ze - zb;  // planes of the launch
        if (what & FEM_SURF) {
            // face columns: one thread per node, consecutive threads along a
            // face (default; 0.19 ms at 384^3 for all surface nodes), or the
            // z-marching column kernel (NB_FEM_FACES=col; 0.22 ms); z-surface
            // planes: one thread per node
            const char *fv = getenv("NB_FEM_FACES");
            const bool faces_node = !(fv && !strcmp(fv, "col"));
            // x-face columns through shared memory (default), unless
            // NB_FEM_FACES=node keeps them in k_fem_surface
            const bool xface = faces_node && !(fv && !strcmp(fv, "node")) && nx >= 2 && ny >= 3;
            const int ncols = faces_node ? 0 : S.ncol_edge;
            if (!faces_node) S.ncol_edge = 0;
            if (xface) {
                S.ncol_edge = 2 * nx;  // fem_edge_col lists the y = 0 and y = ny-1 rows first
                dim3 xg((ny - 2 + XF_Y - 1) / XF_Y, zhi >= 0 ? 2 : (ze - zb + XF_Z - 1) / XF_Z, 2);
                LaunchScope ls(g, xs, "k_fem_surface");
                k_fem_xface<K><<<xg, XF_Y * XF_Z, 0, xs>>>(A, geo, zb, ze, zhi);
            }
            const int64_t n = (int64_t)S.ncol_edge * nzr + (int64_t)S.nin * S.nzs;
            if (n > 0) {
                const int blocks = (int)std::min<int64_t>((n + NB_FSURF_BX - 1) / NB_FSURF_BX, 1 << 30);
                LaunchScope ls(g, ss, "k_fem_surface");
                k_fem_surface<K><<<blocks, NB_FSURF_BX, 0, ss>>>(A, geo, zb, ze, S, zhi);
            }
            if (ncols > 0) {
                if (zhi >= 0) NB_FAIL(NB_EUNSUPPORTED, "plane pairs with the face-column kernel");
                dim3 fg((ncols + 63) / 64, (ze - zb + FZC - 1) / FZC);
                LaunchScope ls(g, ss, "k_fem_faces");
                k_fem_faces<K><<<fg, 64, 0, ss>>>(A, geo, zb, ze, ncols);
            }
        }
        if (!(what & FEM_BULK)) return NB_OK;
        static unsigned attr_set = 0;  // per device: dynamic shared memory above 48 KB
        if (g->device < 32 && !(attr_set & (1u << g->device))) {
            NB_CUDA(cudaFuncSetAttribute(k_fem_tma<K, ZC, NR>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
            attr_set |= 1u << g->device;
        }
        dim3 blk(DOT_TX, DOT_TY / NR);
        if (!conc) {
            LaunchScope ls(g, g->cs, name);
            k_fem_tma<K, ZC, NR><<<dim3(tx, ty, nck), blk, Cfg::SMEM, g->cs>>>(M, A, geo, zb, ze, g->tp, g->T, cm);
        } else {
            NB_CUDA(cudaEventRecord(g->fev[1], ss));  // surface nodes done (x faces: on fs, before the rest)
            {
                FemCtaMap c1 = cm;
                c1.mode = 1;
                LaunchScope ls(g, g->cs, name);
                k_fem_tma<K, ZC, NR><<<dim3(tx - 2, ty - 2, cm.cb - cm.ca + 1), blk, Cfg::SMEM, g->cs>>>(
                    M, A, geo, zb, ze, g->tp, g->T, c1);
                NB_TRY(nb_launch_check(name));
            }
            NB_CUDA(cudaStreamWaitEvent(g->fs, g->fev[1], 0));
            {
                FemCtaMap c2 = cm;
                c2.mode = 2;
                const int n2 = (nck - (cm.cb - cm.ca + 1)) * tx * ty + (cm.cb - cm.ca + 1) * (2 * tx + 2 * (ty - 2));
                LaunchScope ls(g, g->fs, name);
                k_fem_tma<K, ZC, NR><<<n2, blk, Cfg::SMEM, g->fs>>>(M, A, geo, zb, ze, g->tp, g->T, c2);
                NB_TRY(nb_launch_check(name));
            }
            NB_CUDA(cudaEventRecord(g->fev[2], g->fs));
            NB_CUDA(cudaStreamWaitEvent(g->cs, g->fev[2], 0));  // join
        }
    } else {
        constexpr int ZC = 16;
        dim3 blk(DOT_TX, DOT_TY), grd(g->tiles_x, g->tiles_y, (ze - zb + ZC - 1) / ZC);
        LaunchScope ls(g, g->cs, name);
        k_fem_z<K, ZC><<<grd, blk, 0, g->cs>>>(A, geo, zb, ze, g->tp, g->T);
    }
    return nb_launch_check(name);
}

// ===========================================================================
// K u on element-sparse grids.  One
// thread per active node of a 256-cell dot segment (the sparse canonical dot
// order, per component).  The node's 27-neighbourhood comes from the
// nb_sparse_fem_tables mask and row bases; its existing elements (those with
// all 8 nodes active) select the stencil: all 8 and gz >= 2 -> the dense
// interior chain (c_S, structural zeros skipped), otherwise the sparse class
// stencil over the active positions (fem_node_surf_l's chain), gz = 0 ->
// identity row.  A full mask therefore reproduces the dense operator bit for
// bit; general masks are the oracle's element-by-element K (tolerance).
// ===========================================================================
// the interior chain of sp_fem_node: q = 0 .. 26, per q the 9 block
// entries S[q][i][j] = sign * c_cv[class] in (i, j) order, structural zeros
// skipped (fem_cv_class < 0) — bitwise the c_S chain, with every coefficient
// a compile-time constant-bank operand
template <int I, int J, int Q>
__device__ __forceinline__ void sp_fem_cfma(double u, double &acc) {
    constexpr int k = fem_cv_class(Q, I, J);
    if constexpr (k >= 0) acc = fma(fem_cv_sign(Q, I, J) > 0 ? c_cv[k] : -c_cv[k], u, acc);
}
template <int Q, class LD>
__device__ __forceinline__ void sp_fem_interior(const LD &ld, double &acc0, double &acc1, double &acc2) {
    if constexpr (Q < 27) {
        double u0, u1, u2;
        ld(Q, u0, u1, u2);
        sp_fem_cfma<0, 0, Q>(u0, acc0);
        sp_fem_cfma<0, 1, Q>(u1, acc0);
        sp_fem_cfma<0, 2, Q>(u2, acc0);
        sp_fem_cfma<1, 0, Q>(u0, acc1);
        sp_fem_cfma<1, 1, Q>(u1, acc1);
        sp_fem_cfma<1, 2, Q>(u2, acc1);
        sp_fem_cfma<2, 0, Q>(u0, acc2);
        sp_fem_cfma<2, 1, Q>(u1, acc2);
        sp_fem_cfma<2, 2, Q>(u2, acc2);
        sp_fem_interior<Q + 1>(ld, acc0, acc1, acc2);
    }
}

// y_n of an active node off the Dirichlet plane (gz >= 1) from its
// 27-neighbourhood mask m (bit (ox+1) + 3(oy+1) + 9(oz+1)) and a loader
// ld(q, u0, u1, u2) of neighbour q's 3 components (called for the active
// positions in increasing q): the node's existing elements (those with all 8
// nodes active) select the stencil: all 8 and gz >= 2 -> the dense interior
// chain (c_S, structural zeros skipped), otherwise the class stencil of the
// element set (x Dirichlet drop at gz = 1).  Shared by the gather pass and
// the shared-memory box operator, so the two give the same bits.
template <class LD>
__device__ __forceinline__ void sp_fem_node(uint32_t m, int gz, const LD &ld, double (&o)[3]) {
    int em = 0;  // existing elements: corner a of the element at node - off(a)
#pragma unroll
    for (int a = 0; a < 8; ++a) {
        bool ex = true;
#pragma unroll
        for (int b = 0; b < 8; ++b) {
            const int ox = (b & 1) - (a & 1), oy = ((b >> 1) & 1) - ((a >> 1) & 1), oz = ((b >> 2) & 1) - ((a >> 2) & 1);
            ex = ex && ((m >> ((ox + 1) + 3 * (oy + 1) + 9 * (oz + 1))) & 1u);
        }
        em |= ex ? 1 << a : 0;
    }
    const bool drop = gz == 1;
    double acc0 = 0.0, acc1 = 0.0, acc2 = 0.0;
    if (em == 0xff && !drop) {
        // interior: all 27 neighbours active; its own branch keeps the
        // compiler from if-converting the two chains into one predicated
        // sequence (measured: both chains' DFMAs and loads issued per node)
        sp_fem_interior<0>(ld, acc0, acc1, acc2);
    } else {
        const double *C = c_scls + (size_t)(em * 2 + (drop ? 1 : 0)) * 243;
#pragma unroll
        for (int q = 0; q < 27; ++q) {
            if (!((m >> q) & 1u)) continue;
            double u0, u1, u2;
            ld(q, u0, u1, u2);
            const double *K = C + q * 9;
            acc0 = fma(__ldg(K + 0), u0, acc0);
            acc0 = fma(__ldg(K + 1), u1, acc0);
            acc0 = fma(__ldg(K + 2), u2, acc0);
            acc1 = fma(__ldg(K + 3), u0, acc1);
            acc1 = fma(__ldg(K + 4), u1, acc1);
            acc1 = fma(__ldg(K + 5), u2, acc1);
            acc2 = fma(__ldg(K + 6), u0, acc2);
            acc2 = fma(__ldg(K + 7), u1, acc2);
            acc2 = fma(__ldg(K + 8), u2, acc2);
        }
    }
    o[0] = acc0;
    o[1] = acc1;
    o[2] = acc2;
}

struct SpFemArgs {
    const int32_t *seg;
    int64_t seg0, nseg;
    const int64_t *pstart;
    const uint32_t *fm;
    const int32_t *fb;
    int64_t n, hl, cs;
    int gz0, NZ, T;
    double *tp;
    const double *u, *b;
    double *y;
    const CgScal *sc;
};

#ifndef NB_SPF_MINB
#define NB_SPF_MINB 8  // 32 registers: 3.04 ms per K p pass at 384^3 (6: 3.19, unbounded: 3.83)
#endif
template <int KIND>  // 0: y = K u; 1: q = K u, <u, q>; 2: y = b - K u, <y, y>
__global__ void __launch_bounds__(256, NB_SPF_MINB) k_sp_fem(SpFemArgs A) {
    __shared__ double sw[3][8];
    const int t = threadIdx.x;
    const int e = __ldg(A.seg + A.seg0 + blockIdx.x);
    const int zl = e >> 16, sg = e & 0xffff;
    const int64_t j = __ldg(A.pstart + zl) + (int64_t)sg * 256 + t;
    const bool valid = j < __ldg(A.pstart + zl + 1);
    if (KIND == 1 && A.sc->status != 0) return;
    double prod[3] = {0.0, 0.0, 0.0};
    if (valid) {
        const int gz = A.gz0 + zl;
        const int64_t i = A.hl + j;
        double o[3];
        if (gz == 0) {  // Dirichlet identity row
#pragma unroll
            for (int c = 0; c < 3; ++c) o[c] = A.u[c * A.cs + i];
        } else {
            const uint32_t m = __ldg(A.fm + j);
            int32_t base[9];
#pragma unroll
            for (int r = 0; r < 9; ++r) base[r] = __ldg(A.fb + (int64_t)r * A.n + j);
            sp_fem_node(m, gz, [&](int q, double &u0, double &u1, double &u2) {
                const int ox = q % 3 - 1, r = q / 3;
                const uint32_t rb = (m >> (3 * r)) & 7u;
                const int64_t idx = base[r] + __popc(rb & ((1u << (ox + 1)) - 1u));
                u0 = __ldg(A.u + idx), u1 = __ldg(A.u + A.cs + idx), u2 = __ldg(A.u + 2 * A.cs + idx);
            }, o);
        }
#pragma unroll
        for (int c = 0; c < 3; ++c) {
            const int64_t k = c * A.cs + i;
            if (KIND == 2) {
                const double r = __dsub_rn(A.b[k], o[c]);
                A.y[k] = r;
                prod[c] = __dmul_rn(r, r);
            } else {
                A.y[k] = o[c];
                if (KIND == 1) prod[c] = __dmul_rn(A.u[k], o[c]);
            }
        }
    }
    if (KIND == 0) return;
    const int w = t >> 5;
    warp_sums_store<3>(prod, t & 31, &sw[0][w], 8);
    __syncthreads();
    if (t < 3) {
        double s = sw[t][0];
#pragma unroll
        for (int ww = 1; ww < 8; ++ww) s = __dadd_rn(s, sw[t][ww]);
        A.tp[((int64_t)t * A.NZ + A.gz0 + zl) * A.T + sg] = s;
    }
}

nb_status nb_sparse_fem_pass(nb_grid *g, int p, int kind, const int32_t *list, const int32_t *gidx, int64_t s0,
                             int64_t n, const double *u, const double *b, double *y, const CgScal *sc) {
    (void)gidx;
    if (n <= 0) return NB_OK;
    const NbSparsePart &sp = g->sp[p];
    SpFemArgs A{};
    A.seg = list;
    A.seg0 = s0;
    A.nseg = n;
    A.pstart = sp.d_pstart;
    A.fm = sp.d_fm;
    A.fb = sp.d_fb;
    A.n = sp.n;
    A.hl = sp.hl;
    A.cs = sp.cs;
    A.gz0 = g->parts[p].z0;
    A.NZ = g->nz;
    A.T = g->T;
    A.tp = g->tp;
    A.u = u;
    A.b = b;
    A.y = y;
    A.sc = sc;
    const char *name = kind == 0 ? "k_fem_apply" : (kind == 1 ? "k_sp_fem_q" : "k_fem_cg_init");
    LaunchScope ls(g, g->cs, name);
    if (kind == 0)
        k_sp_fem<0><<<(unsigned)n, 256, 0, g->cs>>>(A);
    else if (kind == 1)
        k_sp_fem<1><<<(unsigned)n, 256, 0, g->cs>>>(A);
    else
        k_sp_fem<2><<<(unsigned)n, 256, 0, g->cs>>>(A);
    return nb_launch_check(name);
}


// ---- the sparse FEM operator from shared-memory boxes ----------------------
// The gather pass above issues 81 dependent-address loads per node, nearly
// all L1 misses (the 9 neighbour rows x 3 components of a warp span ~10 KB),
// so it streams ~30x its algorithmic bytes through L2.  Here a CTA owns a
// 32 x 8 tile of a z-chunk (the dense kernels' decomposition of the bounding
// box; only tiles holding an active node are launched) and stages, per
// plane, the 34 x 10 box around the tile x 3 components from the compact
// arrays into a shared-memory ring with 8-byte cp.async (zero-fill for
// inactive cells), together with the box rows' activity bits.  A box cell's
// buffer index is its row word's index plus a popcount (nb_sparse_fem_box_
// tables).  Output plane k is computed when planes k-1 .. k+1 have landed,
// by sp_fem_node over the staged values: the gather pass's arithmetic, so
// the same bits.  Each value is read from DRAM once (ring rows from L2).
#ifndef NB_SFB_NST
#define NB_SFB_NST 5  // ring stages: planes k-1 .. k+1 in use, k+2, k+3 in flight
#endif
#ifndef NB_SFB_ZC
#define NB_SFB_ZC 32  // output planes per CTA
#endif
#ifndef NB_SFB_MINB
#define NB_SFB_MINB 3
#endif
static_assert(NB_SFB_NST >= 5, "the box ring: planes pl-2 .. pl read, pl+1 in flight, pl+2 issued");
#define SFB_W 34
#define SFB_H 10
#define SFB_C (SFB_W * SFB_H)

struct SpFemBoxArgs {
    const int4 *items;
    const uint32_t *rm;
    const int32_t *ri;
    int rw, nx, ny, gz0, nzl;
    int64_t cs;
    const double *u, *b;  // KIND 3: u = the p_new buffer (its halo planes are staged as they are)
    double *y;
    const double *r, *po;  // KIND 3: p_new = r + beta p_old formed while staging own planes
    double *pn, *x;        // KIND 3: p_new and the deferred x += alpha_prev p_old of own nodes
    const CgScal *sc;
    double *tp;            // KIND 1: <u, q> tile partials [3][NZ][T] (dense canonical order)
    int NZ, T, tx;
    int64_t ncell;         // cells of a component's buffer (halo lo + own + halo hi): bulk-copy bound
};

__device__ __forceinline__ void sfb_cp8(double *dst, const double *src, bool on) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(d), "l"(src), "r"(on ? 8 : 0) : "memory");
}

// one staged plane's 9 in-plane positions Q (3 components each, read once
// at compile-time offsets from the node's centre P) applied to the three
// outputs it touches: aA (q = 18 + Q), aB (q = 9 + Q), aC (q = Q)
template <int Q>
__device__ __forceinline__ void sfb_plane(const double *P, double (&aA)[3], double (&aB)[3], double (&aC)[3]) {
    if constexpr (Q < 9) {
        constexpr int e = (Q / 3 - 1) * SFB_W + (Q % 3 - 1);
        const double u0 = P[e], u1 = P[SFB_C + e], u2 = P[2 * SFB_C + e];
        auto blk = [&](auto qc, double (&a)[3]) {
            constexpr int q = decltype(qc)::value;
            sp_fem_cfma<0, 0, q>(u0, a[0]);
            sp_fem_cfma<0, 1, q>(u1, a[0]);
            sp_fem_cfma<0, 2, q>(u2, a[0]);
            sp_fem_cfma<1, 0, q>(u0, a[1]);
            sp_fem_cfma<1, 1, q>(u1, a[1]);
            sp_fem_cfma<1, 2, q>(u2, a[1]);
            sp_fem_cfma<2, 0, q>(u0, a[2]);
            sp_fem_cfma<2, 1, q>(u1, a[2]);
            sp_fem_cfma<2, 2, q>(u2, a[2]);
        };
        blk(std::integral_constant<int, 18 + Q>{}, aA);
        blk(std::integral_constant<int, 9 + Q>{}, aB);
        blk(std::integral_constant<int, Q>{}, aC);
        sfb_plane<Q + 1>(P, aA, aB, aC);
    }
}

// KIND 0: y = K u; 2: y = b - K u; 3 (sparse FEM CG phase A): own planes
// stage r and p_old, every thread turns its own box cells into p_new = r +
// beta p_old (the gather path's map, fma(beta, p_old, r)) right after its
// copies land, so the one barrier per plane still suffices; halo planes stage
// the exchanged p_new.  Each active own node stores p_new and, pending, x +=
// alpha_prev p_old (x loaded a step ahead); interior nodes store q = K p_new.
template <int KIND>
struct SfbCfg {
    static constexpr int NPO = KIND == 3 ? 4 : 0;  // p_old slots: planes pl-1 .. pl+2
    static constexpr int SMEM = (NB_SFB_NST + NPO) * 3 * SFB_C * 8;
};

template <int KIND>
__global__ void __launch_bounds__(256, NB_SFB_MINB) k_sp_fem_box(SpFemBoxArgs A) {
    extern __shared__ __align__(16) double sfb_sm[];
    double(*S)[3][SFB_C] = reinterpret_cast<double(*)[3][SFB_C]>(sfb_sm);
    double(*PO)[3][SFB_C] = reinterpret_cast<double(*)[3][SFB_C]>(sfb_sm + NB_SFB_NST * 3 * SFB_C);
    constexpr int NPO = SfbCfg<KIND>::NPO;
    __shared__ uint64_t RB[NB_SFB_NST][SFB_H];
    __shared__ double sw[2][3][8];  // KIND 1: per output parity, component, tile row
    if (A.sc && A.sc->status != 0) return;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const int4 it = A.items[blockIdx.x];
    const int bxi = it.x & 0x3fffffff;
    const int x0 = bxi * 32, y0 = it.y * 8, zs = it.z, ze = it.w;
    const int np = ze - zs + 2;  // staged planes zs-1 .. ze
    const int nout = ze - zs;
    const int wx = bxi;          // the tile's x word
    const int tile = it.y * A.tx + bxi;
    if (KIND == 1 && (it.x & 0x40000000)) {  // no active node in the tile's chunk: zero partials
        for (int k = tid; k < 3 * nout; k += 256)
            A.tp[((int64_t)(k / nout) * A.NZ + A.gz0 + zs + k % nout) * A.T + tile] = 0.0;
        return;
    }
    // KIND 1: the tile partial of output o (3 components): rows in increasing y
    auto flush = [&](int o) {
        if (tid < 3) {
            const double *v = sw[o & 1][tid];
            double s = v[0];
#pragma unroll
            for (int k = 1; k < 8; ++k) s = __dadd_rn(s, v[k]);
            A.tp[((int64_t)tid * A.NZ + A.gz0 + zs + o) * A.T + tile] = s;
        }
    };
    double beta = 0.0, ap = 0.0;
    bool dox = false;
    if constexpr (KIND == 3) {
        beta = A.sc->beta;
        ap = A.sc->alpha_prev;
        dox = A.sc->pending != 0;
    }
    // Staging is split in two so no thread waits on a table load: fetch(pl)
    // loads plane pl's table words for the thread's (up to 2) box cells and
    // box row into registers one step ahead; issue(pl) turns them into the
    // 8-byte cp.async copies into ring slot pl % NST and the row bits.
    int cx[2], cy[2];
    bool cv[2];
#pragma unroll
    for (int k = 0; k < 2; ++k) {
        const int e = tid + 256 * k;
        cx[k] = x0 - 1 + e % SFB_W;
        cy[k] = y0 - 1 + e / SFB_W;
        cv[k] = e < SFB_C && cx[k] >= 0 && cx[k] < A.nx && cy[k] >= 0 && cy[k] < A.ny;
    }
    // the box rows' bits are built by threads that stage one cell only
    // (tid >= SFB_C - 256 stage one, the others two): balanced plane steps
    const int rt = tid - (SFB_C - 256);  // box row of threads 0 <= rt < SFB_H
    const int ry = y0 - 1 + rt;
    const bool rown = rt >= 0 && rt < SFB_H;
    const bool rv = rown && ry >= 0 && ry < A.ny;
    uint32_t tm[2] = {0u, 0u}, rl = 0u, rm = 0u, rh = 0u;
    int32_t ti[2] = {0, 0};
    auto own = [&](int pl) { const int zl = zs - 1 + pl; return zl >= 0 && zl < A.nzl; };
    auto fetch = [&](int pl) {
        const int64_t row0 = (int64_t)(zs + pl) * A.ny;  // slab row of (zl + 1, y = 0), zl = zs - 1 + pl
#pragma unroll
        for (int k = 0; k < 2; ++k)
            if (cv[k]) {
                const int64_t q = (row0 + cy[k]) * A.rw + (cx[k] >> 5);
                tm[k] = __ldg(A.rm + q);
                ti[k] = __ldg(A.ri + q);
            }
        if (rv) {
            const uint32_t *r = A.rm + (row0 + ry) * A.rw;
            rl = wx > 0 ? __ldg(r + wx - 1) : 0u;
            rm = __ldg(r + wx);
            rh = wx + 1 < A.rw ? __ldg(r + wx + 1) : 0u;
        }
    };
    auto issue = [&](int pl) {
        const int st = pl % NB_SFB_NST;
        const bool form = KIND == 3 && own(pl);
#pragma unroll
        for (int k = 0; k < 2; ++k) {
            const int e = tid + 256 * k;
            if (e < SFB_C) {
                const unsigned b = (unsigned)cx[k] & 31u;
                const bool act = cv[k] && ((tm[k] >> b) & 1u);
                const int64_t idx = act ? ti[k] + __popc(tm[k] & ((1u << b) - 1u)) : 0;
                if (form) {
#pragma unroll
                    for (int c = 0; c < 3; ++c) {
                        sfb_cp8(&S[st][c][e], A.r + c * A.cs + idx, act);
                        sfb_cp8(&PO[pl % (NPO ? NPO : 1)][c][e], A.po + c * A.cs + idx, act);
                    }
                } else {
#pragma unroll
                    for (int c = 0; c < 3; ++c) sfb_cp8(&S[st][c][e], A.u + c * A.cs + idx, act);
                }
            }
        }
        if (rown)  // activity bits of box row rt: bit i = x0 - 1 + i
            RB[st][rt] = rv ? (uint64_t)(rl >> 31) | ((uint64_t)rm << 1) | ((uint64_t)(rh & 1u) << 33) : 0ull;
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    // ring: at step pl (plane pl lands) planes pl-2 .. pl are read (the
    // completed output pl-2 may need all three), pl+1 is in flight and pl+2
    // is issued into the slot of plane pl-3
    constexpr int AHEAD = NB_SFB_NST - 3;
#pragma unroll 1
    for (int pl = 0; pl < AHEAD; ++pl) {
        if (pl < np) {
            fetch(pl);
            issue(pl);
        } else {
            asm volatile("cp.async.commit_group;" ::: "memory");
        }
    }
    if (AHEAD < np) fetch(AHEAD);
    const int x = x0 + lane, y = y0 + w;
    const bool in = x < A.nx && y < A.ny;
    const int ce = (w + 1) * SFB_W + lane + 1;  // the thread's node in a staged box
    const uint32_t lmask = (1u << lane) - 1u;
    // z-march (the dense kernels' scheme): plane pl's 9 positions x 3
    // components are read once and applied to output pl-2 (aA, as its oz =
    // +1 plane), pl-1 (aB, oz = 0) and pl (aC, oz = -1); per output the
    // blocks arrive in q order, so an interior node gets sp_fem_node's
    // interior chain bit for bit.  Output pl-2 is then complete: interior
    // nodes (27 active neighbours, gz >= 2) store aA; every other node is
    // k_sp_fem_list's (so no warp here diverges into a class stencil).
    // The output node's buffer index (row word index + active cells before
    // x) and, for KIND 3, its x are loaded a step ahead.
    double aA[3] = {0.0, 0.0, 0.0}, aB[3] = {0.0, 0.0, 0.0};
    double xo[3] = {0.0, 0.0, 0.0};
    int32_t oi = 0;   // row word index of the next output to be indexed
    int64_t ic = 0;   // buffer index of the output completed next step
#pragma unroll 1
    for (int pl = 0; pl < np; ++pl) {
        asm volatile("cp.async.wait_group %0;" ::"n"(AHEAD - 1) : "memory");
        const int sl = pl % NB_SFB_NST;
        if constexpr (KIND == 3) {
            if (own(pl)) {  // this thread's box cells of plane pl: p_new = r + beta p_old
#pragma unroll
                for (int k = 0; k < 2; ++k) {
                    const int e = tid + 256 * k;
                    if (e < SFB_C)
#pragma unroll
                        for (int c = 0; c < 3; ++c) S[sl][c][e] = fma(beta, PO[pl % NPO][c][e], S[sl][c][e]);
                }
            }
        }
        __syncthreads();  // plane pl landed (p_new formed); plane pl-3's slot is free; sw of output pl-3 written
        if (KIND == 1 && pl >= 3) flush(pl - 3);
        if (pl + AHEAD < np) issue(pl + AHEAD);
        else asm volatile("cp.async.commit_group;" ::: "memory");
        if (pl + AHEAD + 1 < np) fetch(pl + AHEAD + 1);  // lands while this step computes
        double aC[3] = {0.0, 0.0, 0.0};
        // warp-uniform: does the row hold an active node of outputs pl-2 .. pl
        // (centres in planes pl-1 .. pl+1)?  Otherwise the three are never stored
        const uint64_t rows = (pl >= 1 ? RB[(pl + NB_SFB_NST - 1) % NB_SFB_NST][w + 1] : 0ull) | RB[sl][w + 1] |
                              (pl + 1 < np ? RB[(pl + 1) % NB_SFB_NST][w + 1] : 0ull);
        if ((rows >> 1) & 0xffffffffull) sfb_plane<0>(&S[sl][0][ce], aA, aB, aC);
        if (pl >= 2) {
            const int o = pl - 2, zl = zs + o;
            const int s0 = (pl + NB_SFB_NST - 2) % NB_SFB_NST, s1 = (pl + NB_SFB_NST - 1) % NB_SFB_NST;
            const int gz = A.gz0 + zl;
            double prod[3] = {0.0, 0.0, 0.0};
            if (in && ((RB[s1][w + 1] >> (lane + 1)) & 1u)) {
                if constexpr (KIND == 3) {  // every active own node: p_new, deferred x
#pragma unroll
                    for (int c = 0; c < 3; ++c) {
                        __stcs(A.pn + c * A.cs + ic, S[s1][c][ce]);
                        if (dox) __stcs(A.x + c * A.cs + ic, fma(ap, PO[(pl - 1) % NPO][c][ce], xo[c]));
                    }
                }
                // interior iff all 27 neighbours are active (then all 8
                // elements exist) and gz >= 2
                bool full = gz >= 2;
#pragma unroll
                for (int r = 0; r < 9; ++r) {
                    const int oy = r % 3 - 1, oz = r / 3 - 1;
                    const int st = oz < 0 ? s0 : (oz == 0 ? s1 : sl);
                    full = full && ((RB[st][w + 1 + oy] >> lane) & 7u) == 7u;
                }
                if (full) {
#pragma unroll
                    for (int c = 0; c < 3; ++c) {
                        const int64_t kk = c * A.cs + ic;
                        A.y[kk] = KIND == 2 ? __dsub_rn(A.b[kk], aA[c]) : aA[c];
                    }
                }
                if constexpr (KIND == 1) {  // <u, q>: the list kernel's q for the other nodes (it ran first)
#pragma unroll
                    for (int c = 0; c < 3; ++c)
                        prod[c] = __dmul_rn(S[s1][c][ce], full ? aA[c] : __ldcs(A.y + c * A.cs + ic));
                }
            }
            if constexpr (KIND == 1) {  // the tile row's 3 canonical warp sums
                const double v = warp_sum_multi<3>(prod, lane);
                const int i = warp_multi_index<3>(lane);
                if (i < 3 && (lane & (32 / WarpMulti<3>::M - 1)) == 0) sw[o & 1][i][w] = v;
            }
        }
        // the next output (pl - 1, centre plane pl): its buffer index and x
        if (pl >= 1 && pl - 1 < nout) {
            const uint64_t cb = RB[sl][w + 1];
            ic = oi + __popc((uint32_t)(cb >> 1) & lmask);
            if constexpr (KIND == 3)
                if (dox && in && ((cb >> (lane + 1)) & 1u))
#pragma unroll
                    for (int c = 0; c < 3; ++c) xo[c] = __ldcs(A.x + c * A.cs + ic);
        }
        // and the row word index of output pl (centre plane pl + 1)
        if (in && pl < nout) oi = __ldg(A.ri + ((int64_t)(zs + pl + 1) * A.ny + y) * A.rw + wx);
#pragma unroll
        for (int c = 0; c < 3; ++c) {
            aA[c] = aB[c];
            aB[c] = aC[c];
        }
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    if constexpr (KIND == 1) {  // the last output's partials (the one before was flushed in the loop)
        __syncthreads();
        flush(nout - 1);
    }
}

// mbarrier arrivals of the warp-specialised box kernel below
__device__ __forceinline__ void sfw_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void sfw_cp_arrive(uint64_t *bar) {
    asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// Warp-specialised, two-row variant of k_sp_fem_box for kinds 0 / 2
// (default; NB_SFB_NR1=1 selects the kernel above).  Four producer warps
// stage the planes (table words loaded one plane ahead, 8-byte cp.async,
// row bits) up to NB_SF2_NST planes ahead and signal each slot through an
// mbarrier (cp.async.mbarrier.arrive.noinc, plus a release arrive by the
// row-bit writers); eight consumer warps run the z-march and release a slot
// (one arrive per warp) after its last read — no CTA barrier in the plane
// loop.  A consumer thread owns two rows of a 32 x 16 tile (box 34 x 18):
// per plane it loads box rows ra-1 .. ra+2 of the three columns once (36
// values for its 2 nodes instead of 54: the middle rows are kept in
// registers from one row of positions to the next) and applies each
// position's blocks in the same q order per node — the same bits.
// Measured (round 2b, 384^3 full cube, CG iteration): 3.23 ms against 3.26
// for the single-role kernel; a one-row warp-specialised version: 3.29.
#ifndef NB_SF2_NST
#define NB_SF2_NST 6
#endif
#define SF2_H 18
#ifndef NB_SF2_SLEEP_NS
#define NB_SF2_SLEEP_NS 256
#endif
#define SF2_C (SFB_W * SF2_H)
#define SF2_PT 128
#define SF2_SMEM (NB_SF2_NST * 3 * SF2_C * 8)
#define SF2B_SMEM (NB_SF2_NST * 3 * 36 * SF2_H * 8)

template <int q>
__device__ __forceinline__ void sf2_blk(double u0, double u1, double u2, double (&a)[3]) {
    sp_fem_cfma<0, 0, q>(u0, a[0]);
    sp_fem_cfma<0, 1, q>(u1, a[0]);
    sp_fem_cfma<0, 2, q>(u2, a[0]);
    sp_fem_cfma<1, 0, q>(u0, a[1]);
    sp_fem_cfma<1, 1, q>(u1, a[1]);
    sp_fem_cfma<1, 2, q>(u2, a[1]);
    sp_fem_cfma<2, 0, q>(u0, a[2]);
    sp_fem_cfma<2, 1, q>(u1, a[2]);
    sp_fem_cfma<2, 2, q>(u2, a[2]);
}
// position Q of the plane for both rows: row 0 takes values v0, row 1 v1
template <int Q>
__device__ __forceinline__ void sf2_pos(const double (&v0)[3], const double (&v1)[3], double (&aA)[2][3],
                                        double (&aB)[2][3], double (&aC)[2][3]) {
    sf2_blk<18 + Q>(v0[0], v0[1], v0[2], aA[0]);
    sf2_blk<9 + Q>(v0[0], v0[1], v0[2], aB[0]);
    sf2_blk<Q>(v0[0], v0[1], v0[2], aC[0]);
    sf2_blk<18 + Q>(v1[0], v1[1], v1[2], aA[1]);
    sf2_blk<9 + Q>(v1[0], v1[1], v1[2], aB[1]);
    sf2_blk<Q>(v1[0], v1[1], v1[2], aC[1]);
}
// R0 .. R3 = the thread's column (component 0) in box rows ra-1 .. ra+2 of
// the plane; CS = the component stride of the slot
template <int CS>
__device__ __forceinline__ void sf2_plane(const double *R0, const double *R1, const double *R2, const double *R3,
                                          double (&aA)[2][3], double (&aB)[2][3], double (&aC)[2][3]) {
    double keep[3][3], v0[3], v1[3];
#define SF2_LD(v, R, ox)                                 \
    {                                                    \
        const double *pp = (R) + (ox);                   \
        v[0] = pp[0], v[1] = pp[CS], v[2] = pp[2 * CS];  \
    }
    // oy = -1: rows ra-1 (node 0), ra (node 1, kept)
    SF2_LD(v0, R0, -1) SF2_LD(v1, R1, -1) keep[0][0] = v1[0], keep[0][1] = v1[1], keep[0][2] = v1[2];
    sf2_pos<0>(v0, v1, aA, aB, aC);
    SF2_LD(v0, R0, 0) SF2_LD(v1, R1, 0) keep[1][0] = v1[0], keep[1][1] = v1[1], keep[1][2] = v1[2];
    sf2_pos<1>(v0, v1, aA, aB, aC);
    SF2_LD(v0, R0, 1) SF2_LD(v1, R1, 1) keep[2][0] = v1[0], keep[2][1] = v1[1], keep[2][2] = v1[2];
    sf2_pos<2>(v0, v1, aA, aB, aC);
    // oy = 0: rows ra (kept), ra+1 (node 1, kept next)
#pragma unroll
    for (int ox = 0; ox < 3; ++ox) {
        SF2_LD(v1, R2, ox - 1)
        v0[0] = keep[ox][0], v0[1] = keep[ox][1], v0[2] = keep[ox][2];
        keep[ox][0] = v1[0], keep[ox][1] = v1[1], keep[ox][2] = v1[2];
        if (ox == 0) sf2_pos<3>(v0, v1, aA, aB, aC);
        if (ox == 1) sf2_pos<4>(v0, v1, aA, aB, aC);
        if (ox == 2) sf2_pos<5>(v0, v1, aA, aB, aC);
    }
    // oy = +1: rows ra+1 (kept), ra+2
#pragma unroll
    for (int ox = 0; ox < 3; ++ox) {
        SF2_LD(v1, R3, ox - 1)
        v0[0] = keep[ox][0], v0[1] = keep[ox][1], v0[2] = keep[ox][2];
        if (ox == 0) sf2_pos<6>(v0, v1, aA, aB, aC);
        if (ox == 1) sf2_pos<7>(v0, v1, aA, aB, aC);
        if (ox == 2) sf2_pos<8>(v0, v1, aA, aB, aC);
    }
#undef SF2_LD
}

// producers wait for a free slot with a back-off: their spinning took issue
// slots from the consumers (ncu: ~15 try_wait executions per node)
__device__ __forceinline__ void sf2_wait_empty(uint64_t *bar, uint32_t parity) {
    uint32_t done;
    for (;;) {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
        if (done) return;
        __nanosleep(NB_SF2_SLEEP_NS);
    }
}

// one bulk copy (TMA engine) of `bytes` global -> shared, completing on bar
__device__ __forceinline__ void sf2_bulk(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

// BULK: box rows whose 34-cell window is fully active (a contiguous index
// range) arrive as one bulk copy per component (cp.async.bulk, 272 or 288
// bytes: an odd first index starts one cell earlier for 16-byte alignment,
// the row's shift kept in bit 40 of its row bits) into 36-wide rows; the
// other rows cell by cell as above.  Inactive box cells are not copied at
// all (an interior node reads active cells only).
template <int KIND, bool BULK>  // KIND 0: y = K u; 2: y = b - K u
__global__ void __launch_bounds__(256 + SF2_PT, 2) k_sp_fem_box2(SpFemBoxArgs A) {
    constexpr int RS = BULK ? 36 : SFB_W;  // box row stride
    constexpr int C = RS * SF2_H;          // component stride of a slot
    extern __shared__ __align__(16) double sf2_sm[];
    double(*S)[3][C] = reinterpret_cast<double(*)[3][C]>(sf2_sm);
    __shared__ uint64_t RB[NB_SF2_NST][SF2_H];
    __shared__ __align__(8) uint64_t full[NB_SF2_NST], empty[NB_SF2_NST];
    if (A.sc && A.sc->status != 0) return;
    const int tid = threadIdx.x;
    const int4 it = A.items[blockIdx.x];
    const int bxi = it.x & 0x3fffffff;
    const int x0 = bxi * 32, y0 = it.y * 16, zs = it.z, ze = it.w;
    const int np = ze - zs + 2;
    const int nout = ze - zs;
    const int wx = bxi;
    if (tid == 0) {
        for (int k = 0; k < NB_SF2_NST; ++k) {
            mbar_init(&full[k], SF2_PT + (BULK ? SF2_PT / 32 : SF2_H));
            mbar_init(&empty[k], 8);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (tid >= 256) {  // ---- producers ----
      if constexpr (BULK) {
        // warp pw stages box rows pw, pw + 4, ... (<= 5): lane 6 r + k loads
        // word k of row r's three rm and three ri words, one plane ahead,
        // and the warp shares them by shuffles; then one bulk copy per
        // component (lanes 0-2) if a row's window is fully active, else
        // cell by cell
        const int pw = (tid - 256) >> 5, pl_ = tid & 31;
        constexpr int NRW = (SF2_H + SF2_PT / 32 - 1) / (SF2_PT / 32);  // rows per producer warp
        auto load_w = [&](int q) -> uint32_t {
            const int r = pl_ / 6, k = pl_ % 6, j = pw + (SF2_PT / 32) * r, yy = y0 - 1 + j;
            const int wd = wx - 1 + k % 3;
            uint32_t v = 0u;
            if (r < NRW && j < SF2_H && yy >= 0 && yy < A.ny && wd >= 0 && wd < A.rw) {
                const int64_t kk = ((int64_t)(zs + q) * A.ny + yy) * A.rw + wd;
                v = k < 3 ? __ldg(A.rm + kk) : (uint32_t)__ldg(A.ri + kk);
            }
            return v;
        };
        uint32_t wcur = load_w(0);
#pragma unroll 1
        for (int q = 0; q < np; ++q) {
            const int st = q % NB_SF2_NST;
            const uint32_t wnext = q + 1 < np ? load_w(q + 1) : 0u;
            if (q >= NB_SF2_NST) sf2_wait_empty(&empty[st], (uint32_t)((q / NB_SF2_NST) - 1) & 1u);
#pragma unroll
            for (int r = 0; r < NRW; ++r) {
                const int j = pw + (SF2_PT / 32) * r;
                const uint32_t m0 = __shfl_sync(0xffffffffu, wcur, 6 * r), m1 = __shfl_sync(0xffffffffu, wcur, 6 * r + 1),
                               m2 = __shfl_sync(0xffffffffu, wcur, 6 * r + 2);
                const int32_t i0 = (int32_t)__shfl_sync(0xffffffffu, wcur, 6 * r + 3),
                              i1 = (int32_t)__shfl_sync(0xffffffffu, wcur, 6 * r + 4),
                              i2 = (int32_t)__shfl_sync(0xffffffffu, wcur, 6 * r + 5);
                if (j >= SF2_H) break;
                const uint64_t bits = (uint64_t)(m0 >> 31) | ((uint64_t)m1 << 1) | ((uint64_t)(m2 & 1u) << 33);
                uint64_t sh = 0;
                const int64_t idx0 = i0 + __popc(m0 & 0x7fffffffu);  // cell x0 - 1 (if active)
                // a full window; an odd first index copies one cell more on
                // each side, which must stay inside the component's cells
                if (bits == (1ull << 34) - 1ull && (!(idx0 & 1) || idx0 + 34 < A.ncell)) {
                    sh = (uint64_t)(idx0 & 1);
                    if (pl_ < 3)
                        sf2_bulk(&S[st][pl_][j * RS], A.u + pl_ * A.cs + idx0 - (int64_t)sh, sh ? 288u : 272u,
                                 &full[st]);
                } else {
#pragma unroll
                    for (int h = 0; h < 2; ++h) {
                        const int i = pl_ + 32 * h;  // window cell x0 - 1 + i
                        if (i < SFB_W && ((bits >> i) & 1u)) {
                            const uint32_t m = i == 0 ? m0 : (i == 33 ? m2 : m1);
                            const int32_t ib = i == 0 ? i0 : (i == 33 ? i2 : i1);
                            const unsigned b = i == 0 ? 31u : (i == 33 ? 0u : (unsigned)(i - 1));
                            const int64_t idx = ib + __popc(m & ((1u << b) - 1u));
#pragma unroll
                            for (int c = 0; c < 3; ++c) sfb_cp8(&S[st][c][j * RS + i], A.u + c * A.cs + idx, true);
                        }
                    }
                }
                if (pl_ == 0) RB[st][j] = bits | (sh << 40);
            }
            wcur = wnext;
            sfw_cp_arrive(&full[st]);  // this thread's cell copies (bulk copies count bytes)
            __syncwarp();
            if (pl_ == 0) sfw_arrive(&full[st]);  // after the warp's row bits
        }
        asm volatile("cp.async.wait_all;" ::: "memory");
        return;
      } else {
        // a plane's table words are loaded one plane ahead (two register
        // sets), so the copies of plane q issue while plane q+1's words fly
        const int pt = tid - 256;
        constexpr int NC = (SF2_C + SF2_PT - 1) / SF2_PT;
        const int ry = y0 - 1 + pt;
        const bool rown = pt < SF2_H, rv = rown && ry >= 0 && ry < A.ny;
        auto load_words = [&](int q, uint32_t (&tm)[NC + 3], int32_t (&ti)[NC]) {
            const int64_t row0 = (int64_t)(zs + q) * A.ny;  // slab row of (zl + 1, y = 0), zl = zs - 1 + q
#pragma unroll
            for (int k = 0; k < NC; ++k) {
                const int e = pt + SF2_PT * k;
                const int x = x0 - 1 + e % SFB_W, yy = y0 - 1 + e / SFB_W;
                tm[k] = 0u;
                ti[k] = 0;
                if (e < SF2_C && x >= 0 && x < A.nx && yy >= 0 && yy < A.ny) {
                    const int64_t kk = (row0 + yy) * A.rw + (x >> 5);
                    tm[k] = __ldg(A.rm + kk);
                    ti[k] = __ldg(A.ri + kk);
                }
            }
            tm[NC] = tm[NC + 1] = tm[NC + 2] = 0u;
            if (rv) {  // the row bits' three words
                const uint32_t *r = A.rm + (row0 + ry) * A.rw;
                tm[NC] = wx > 0 ? __ldg(r + wx - 1) : 0u;
                tm[NC + 1] = __ldg(r + wx);
                tm[NC + 2] = wx + 1 < A.rw ? __ldg(r + wx + 1) : 0u;
            }
        };
        auto issue_plane = [&](int q, const uint32_t (&tm)[NC + 3], const int32_t (&ti)[NC]) {
            const int st = q % NB_SF2_NST;
            if (q >= NB_SF2_NST) sf2_wait_empty(&empty[st], (uint32_t)((q / NB_SF2_NST) - 1) & 1u);
#pragma unroll
            for (int k = 0; k < NC; ++k) {
                const int e = pt + SF2_PT * k;
                if (e < SF2_C) {
                    const unsigned b = (unsigned)(x0 - 1 + e % SFB_W) & 31u;
                    const bool act = (tm[k] >> b) & 1u;
                    const int64_t idx = act ? ti[k] + __popc(tm[k] & ((1u << b) - 1u)) : 0;
#pragma unroll
                    for (int c = 0; c < 3; ++c) sfb_cp8(&S[st][c][e], A.u + c * A.cs + idx, act);
                }
            }
            sfw_cp_arrive(&full[st]);
            if (rown) {
                RB[st][pt] = (uint64_t)(tm[NC] >> 31) | ((uint64_t)tm[NC + 1] << 1) |
                             ((uint64_t)(tm[NC + 2] & 1u) << 33);
                sfw_arrive(&full[st]);
            }
        };
        uint32_t tA[NC + 3], tB[NC + 3];
        int32_t iA[NC], iB[NC];
        load_words(0, tA, iA);
#pragma unroll 1
        for (int q = 0; q < np; q += 2) {
            if (q + 1 < np) load_words(q + 1, tB, iB);
            issue_plane(q, tA, iA);
            if (q + 1 >= np) break;
            if (q + 2 < np) load_words(q + 2, tA, iA);
            issue_plane(q + 1, tB, iB);
        }
        asm volatile("cp.async.wait_all;" ::: "memory");
        return;
      }
    }
    // ---- consumers: rows ra = y0 + 2w and ra + 1 ----
    const int lane = tid & 31, w = tid >> 5;
    const int x = x0 + lane, ya = y0 + 2 * w;
    const bool xin = x < A.nx;
    const int c0 = 2 * w * RS + lane + 1;  // the thread's column in box row ra - 1
    const uint32_t lmask = (1u << lane) - 1u;
    double aA[2][3] = {}, aB[2][3] = {};
    int32_t oi[2] = {0, 0};
    int64_t ic[2] = {0, 0};
    double bo[2][3] = {};  // KIND 2: b of the output completed next step
    mbar_wait(&full[0], 0u);
#pragma unroll 1
    for (int pl = 0; pl < np; ++pl) {
        const int sl = pl % NB_SF2_NST;
        if (pl + 1 < np) mbar_wait(&full[(pl + 1) % NB_SF2_NST], (uint32_t)((pl + 1) / NB_SF2_NST) & 1u);
        double aC[2][3] = {};
        const int sm1 = (pl + NB_SF2_NST - 1) % NB_SF2_NST, sp1 = (pl + 1) % NB_SF2_NST;
        const uint64_t rows = (pl >= 1 ? RB[sm1][2 * w + 1] | RB[sm1][2 * w + 2] : 0ull) | RB[sl][2 * w + 1] |
                              RB[sl][2 * w + 2] | (pl + 1 < np ? RB[sp1][2 * w + 1] | RB[sp1][2 * w + 2] : 0ull);
        if ((rows >> 1) & 0xffffffffull) {
            const double *P = &S[sl][0][c0];
            if constexpr (BULK) {  // each row at its shift
                const int b0 = 2 * w;
                sf2_plane<C>(P + ((RB[sl][b0] >> 40) & 1), P + RS + ((RB[sl][b0 + 1] >> 40) & 1),
                             P + 2 * RS + ((RB[sl][b0 + 2] >> 40) & 1), P + 3 * RS + ((RB[sl][b0 + 3] >> 40) & 1),
                             aA, aB, aC);
            } else {
                sf2_plane<C>(P, P + RS, P + 2 * RS, P + 3 * RS, aA, aB, aC);
            }
        }
        if (pl >= 2) {
            const int o = pl - 2, zl = zs + o;
            const int s0 = (pl + NB_SF2_NST - 2) % NB_SF2_NST, s1 = sm1;
            const int gz = A.gz0 + zl;
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const int br = 2 * w + r + 1;  // the node's box row
                if (xin && ya + r < A.ny && ((RB[s1][br] >> (lane + 1)) & 1u)) {
                    bool full_nb = gz >= 2;
#pragma unroll
                    for (int k = 0; k < 9; ++k) {
                        const int oy = k % 3 - 1, oz = k / 3 - 1;
                        const int st = oz < 0 ? s0 : (oz == 0 ? s1 : sl);
                        full_nb = full_nb && ((RB[st][br + oy] >> lane) & 7u) == 7u;
                    }
                    if (full_nb) {
#pragma unroll
                        for (int c = 0; c < 3; ++c) {
                            const int64_t kk = c * A.cs + ic[r];
                            A.y[kk] = KIND == 2 ? __dsub_rn(bo[r][c], aA[r][c]) : aA[r][c];
                        }
                    }
                }
            }
        }
        if (pl >= 1 && pl - 1 < nout) {  // the next output's (centre plane pl) buffer indices
#pragma unroll
            for (int r = 0; r < 2; ++r) ic[r] = oi[r] + __popc((uint32_t)(RB[sl][2 * w + r + 1] >> 1) & lmask);
            if constexpr (KIND == 2) {  // b of the next output, a step ahead (set-up only)
#pragma unroll
                for (int r = 0; r < 2; ++r)
                    if (xin && ya + r < A.ny && ((RB[sl][2 * w + r + 1] >> (lane + 1)) & 1u))
#pragma unroll
                        for (int c = 0; c < 3; ++c) bo[r][c] = __ldg(A.b + c * A.cs + ic[r]);
            }
        }
        if (xin && pl < nout) {
#pragma unroll
            for (int r = 0; r < 2; ++r)
                if (ya + r < A.ny) oi[r] = __ldg(A.ri + ((int64_t)(zs + pl + 1) * A.ny + ya + r) * A.rw + wx);
        }
#pragma unroll
        for (int r = 0; r < 2; ++r)
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                aA[r][c] = aB[r][c];
                aB[r][c] = aC[r][c];
            }
        if (pl >= 2) {
            __syncwarp();
            if (lane == 0) sfw_arrive(&empty[(pl - 2) % NB_SF2_NST]);
        }
    }
}

// The non-interior active nodes of the box operator (element set not full,
// gz <= 1; ~2 % of a cube's nodes): one thread per node of the host-built
// list {buffer index, gz, 27-neighbourhood mask, 9 row bases} (the gather
// pass's per-node inputs), same sp_fem_node arithmetic.
struct SpFemNode {
    int32_t i, gz;
    uint32_t m;
    int32_t base[9];
};
static_assert(sizeof(SpFemNode) == 48, "three 16-byte loads per node");

template <int KIND>  // 0: y = K u; 2: y = b - K u
__global__ void __launch_bounds__(128) k_sp_fem_list(const SpFemNode *__restrict__ L, int64_t n0, int64_t n1,
                                                    int64_t cs, const double *__restrict__ u,
                                                    const double *__restrict__ b, double *y, const CgScal *sc) {
    if (sc && sc->status != 0) return;
    const int64_t t = n0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= n1) return;
    const SpFemNode nd = L[t];
    double o[3];
    if (nd.gz == 0) {  // Dirichlet identity row
#pragma unroll
        for (int c = 0; c < 3; ++c) o[c] = u[c * cs + nd.i];
    } else {
        const uint32_t m = nd.m;
        sp_fem_node(m, nd.gz, [&](int q, double &u0, double &u1, double &u2) {
            const int ox = q % 3 - 1, r = q / 3;
            const uint32_t rb = (m >> (3 * r)) & 7u;
            const int64_t idx = nd.base[r] + __popc(rb & ((1u << (ox + 1)) - 1u));
            u0 = __ldg(u + idx), u1 = __ldg(u + cs + idx), u2 = __ldg(u + 2 * cs + idx);
        }, o);
    }
#pragma unroll
    for (int c = 0; c < 3; ++c) {
        const int64_t k = c * cs + nd.i;
        y[k] = KIND == 2 ? __dsub_rn(b[k], o[c]) : o[c];
    }
}

// per-segment partials of <a, b> (3 components): k_sp_fem's dot, bit for bit
__global__ void __launch_bounds__(256) k_sp_fem_dot(const int32_t *__restrict__ seg, const int64_t *__restrict__ pstart,
                                                   int64_t hl, int64_t cs, int gz0, int NZ, int T, double *tp,
                                                   const double *__restrict__ a, const double *__restrict__ b,
                                                   const CgScal *sc) {
    __shared__ double sw[3][8];
    const int t = threadIdx.x;
    const int e = __ldg(seg + blockIdx.x);
    const int zl = e >> 16, sg = e & 0xffff;
    const int64_t j = __ldg(pstart + zl) + (int64_t)sg * 256 + t;
    const bool valid = j < __ldg(pstart + zl + 1);
    if (sc && sc->status != 0) return;
    double prod[3] = {0.0, 0.0, 0.0};
    if (valid) {
        const int64_t i = hl + j;
#pragma unroll
        for (int c = 0; c < 3; ++c) prod[c] = __dmul_rn(__ldcs(a + c * cs + i), __ldcs(b + c * cs + i));
    }
    const int w = t >> 5;
    warp_sums_store<3>(prod, t & 31, &sw[0][w], 8);
    __syncthreads();
    if (t < 3) {
        double s = sw[t][0];
#pragma unroll
        for (int ww = 1; ww < 8; ++ww) s = __dadd_rn(s, sw[t][ww]);
        tp[((int64_t)t * NZ + gz0 + zl) * T + sg] = s;
    }
}

bool nb_sparse_fem_boxed() { return !getenv("NB_SPF_GATHER"); }

nb_status nb_sparse_fem_box(nb_grid *g, int p, int kind, const std::vector<int> &ranges, const double *u,
                            const double *b, double *y, const CgScal *sc, const SpFemCgA *cga) {
    const int4 *items = nullptr;
    int64_t n = 0;
    NB_TRY(nb_sparse_fem_box_list(g, p, ranges, NB_SFB_ZC, &items, &n, kind == 1));
    const NbSparsePart &sp = g->sp[p];
    SpFemBoxArgs A{};
    A.items = items;
    A.rm = sp.d_rm;
    A.ri = sp.d_ri;
    A.rw = sp.rw;
    A.nx = g->nx;
    A.ny = g->ny;
    A.gz0 = g->parts[p].z0;
    A.nzl = g->parts[p].nz();
    A.u = u;
    A.b = b;
    A.y = y;
    A.sc = sc;
    A.cs = sp.cs;
    A.ncell = sp.hl + sp.n + sp.hh;
    if (kind == 1) {  // <u, q> in tile order: the caller swaps sp_tp in for the finalize
        NB_TRY(nb_sparse_tile_tp(g));
        A.tp = g->sp_tp;
        A.T = g->sp_T;
        A.NZ = g->nz;
        A.tx = (g->nx + 31) / 32;
    }
    if (kind == 3) {
        if (!cga || !sc) NB_FAIL(NB_EINVAL, "sparse FEM phase A needs the CG buffers");
        A.r = cga->r;
        A.po = cga->po;
        A.pn = cga->pn;
        A.x = cga->x;
        A.u = cga->pn;  // halo planes: the exchanged p_new
    }
    const char *name = kind == 2 ? "k_fem_cg_init" : kind == 3 ? "k_sp_fem_cg_a" : (sc ? "k_sp_fem_q" : "k_fem_apply");
    // the list nodes (kinds 0 / 2 read only the input) run on the side
    // stream concurrently with the box kernel, which leaves the SMs room
    // (the list kernel is latency-bound: 11-18 % issue alone); kind 1 reads
    // their q for the dot, so they run first; kind 3 reads the box kernel's
    // p_new and runs after it
    bool any_list = false;
    for (size_t r = 0; r + 1 < ranges.size(); r += 2)
        any_list |= sp.fnode_start[ranges[r + 1]] > sp.fnode_start[ranges[r]];
    const bool conc = any_list && (kind == 0 || kind == 2) && !getenv("NB_SPF_SERIAL");
    cudaStream_t ls_stream = g->cs;
    if (conc) {
        if (!g->fs) {
            int lo, hi;
            NB_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
            NB_CUDA(cudaStreamCreateWithPriority(&g->fs, cudaStreamNonBlocking, hi));
            for (auto &e : g->fev) NB_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        }
        NB_CUDA(cudaEventRecord(g->fev[0], g->cs));  // fork
        NB_CUDA(cudaStreamWaitEvent(g->fs, g->fev[0], 0));
        ls_stream = g->fs;
    }
    auto lists = [&](int lk, const double *lu) -> nb_status {
        // the ranges' non-interior nodes (contiguous per range: the list is in plane order)
        for (size_t r = 0; r + 1 < ranges.size(); r += 2) {
            const int64_t a = sp.fnode_start[ranges[r]], e = sp.fnode_start[ranges[r + 1]];
            if (e <= a) continue;
            const SpFemNode *L = (const SpFemNode *)sp.d_fnode;
            const unsigned nb = (unsigned)((e - a + 127) / 128);
            LaunchScope ls(g, ls_stream, name);
            if (lk == 2)
                k_sp_fem_list<2><<<nb, 128, 0, ls_stream>>>(L, a, e, sp.cs, lu, b, y, sc);
            else
                k_sp_fem_list<0><<<nb, 128, 0, ls_stream>>>(L, a, e, sp.cs, lu, b, y, sc);
            NB_TRY(nb_launch_check(name));
        }
        return NB_OK;
    };
    if (kind == 1) NB_TRY(lists(0, u));
    if (n > 0) {
        static unsigned attr_set = 0;  // per device: dynamic shared memory above 48 KB
        if (g->device >= 32 || !(attr_set & (1u << g->device))) {
            NB_CUDA(cudaFuncSetAttribute(k_sp_fem_box<0>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         SfbCfg<0>::SMEM));
            NB_CUDA(cudaFuncSetAttribute(k_sp_fem_box<1>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         SfbCfg<1>::SMEM));
            NB_CUDA(cudaFuncSetAttribute(k_sp_fem_box<2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         SfbCfg<2>::SMEM));
            NB_CUDA(cudaFuncSetAttribute(k_sp_fem_box<3>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         SfbCfg<3>::SMEM));
            if (g->device < 32) attr_set |= 1u << g->device;
        }
        static unsigned ws_attr = 0;
        const bool nr2 = (kind == 0 || kind == 2) && !getenv("NB_SFB_NR1");
        const bool bulk = !getenv("NB_SFB_NOBULK");
        const int4 *items2 = nullptr;
        int64_t n2 = 0;
        SpFemBoxArgs A2 = A;
        if (nr2) {  // 32 x 16 tiles
            NB_TRY(nb_sparse_fem_box_list(g, p, ranges, NB_SFB_ZC, &items2, &n2, false, 16));
            A2.items = items2;
        }
        if (nr2 && (g->device >= 32 || !(ws_attr & (1u << g->device)))) {
            NB_CUDA(cudaFuncSetAttribute(k_sp_fem_box2<0, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, SF2_SMEM));
            NB_CUDA(cudaFuncSetAttribute(k_sp_fem_box2<2, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, SF2_SMEM));
            NB_CUDA(cudaFuncSetAttribute(k_sp_fem_box2<0, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, SF2B_SMEM));
            NB_CUDA(cudaFuncSetAttribute(k_sp_fem_box2<2, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, SF2B_SMEM));
            if (g->device < 32) ws_attr |= 1u << g->device;
        }
        LaunchScope ls(g, g->cs, name);
        if (nr2 && bulk && kind == 2)
            k_sp_fem_box2<2, true><<<(unsigned)n2, 256 + SF2_PT, SF2B_SMEM, g->cs>>>(A2);
        else if (nr2 && bulk)
            k_sp_fem_box2<0, true><<<(unsigned)n2, 256 + SF2_PT, SF2B_SMEM, g->cs>>>(A2);
        else if (nr2 && kind == 2)
            k_sp_fem_box2<2, false><<<(unsigned)n2, 256 + SF2_PT, SF2_SMEM, g->cs>>>(A2);
        else if (nr2)
            k_sp_fem_box2<0, false><<<(unsigned)n2, 256 + SF2_PT, SF2_SMEM, g->cs>>>(A2);
        else if (kind == 2)
            k_sp_fem_box<2><<<(unsigned)n, 256, SfbCfg<2>::SMEM, g->cs>>>(A);
        else if (kind == 3)
            k_sp_fem_box<3><<<(unsigned)n, 256, SfbCfg<3>::SMEM, g->cs>>>(A);
        else if (kind == 1)
            k_sp_fem_box<1><<<(unsigned)n, 256, SfbCfg<1>::SMEM, g->cs>>>(A);
        else
            k_sp_fem_box<0><<<(unsigned)n, 256, SfbCfg<0>::SMEM, g->cs>>>(A);
        NB_TRY(nb_launch_check(name));
    }
    if (kind == 0 || kind == 2) NB_TRY(lists(kind, u));
    if (kind == 3) NB_TRY(lists(0, cga->pn));  // the list nodes' q = K p_new reads the stored p_new
    if (conc) {
        NB_CUDA(cudaEventRecord(g->fev[2], g->fs));
        NB_CUDA(cudaStreamWaitEvent(g->cs, g->fev[2], 0));  // join
    }
    return NB_OK;
}

nb_status nb_sparse_fem_dot(nb_grid *g, int p, const double *a, const double *b, const CgScal *sc) {
    const NbSparsePart &sp = g->sp[p];
    const int64_t nseg = sp.seg_start.back();
    if (nseg <= 0) return NB_OK;
    LaunchScope ls(g, g->cs, "k_sp_fem_dot");
    k_sp_fem_dot<<<(unsigned)nseg, 256, 0, g->cs>>>(sp.d_seg, sp.d_pstart, sp.hl, sp.cs, g->parts[p].z0, g->nz, g->T,
                                                    g->tp, a, b, sc);
    return nb_launch_check("k_sp_fem_dot");
}

// local plane ranges of partition p: 0 = all, 1 = the interior (planes whose
// neighbours are own planes), 2 = the boundary planes facing a neighbour
static std::vector<int> sp_box_ranges(const nb_grid *g, int p, int which) {
    const NbPart &q = g->parts[p];
    const int nz = q.nz();
    if (which == 0) return {0, nz};
    const int ib = q.lo >= 0 ? 1 : 0, ie = std::max(ib, nz - (q.hi >= 0 ? 1 : 0));
    if (which == 1) return {ib, ie};
    std::vector<int> r;
    if (q.lo >= 0) r.insert(r.end(), {0, 1});
    if (q.hi >= 0 && ie < nz) r.insert(r.end(), {nz - 1, nz});
    return r;
}

nb_status nb_sparse_fem_box_ranges(nb_grid *g, int p, int which, const double *u, const double *b, double *y,
                                   const CgScal *sc, int kind, const SpFemCgA *cga) {
    return nb_sparse_fem_box(g, p, kind, sp_box_ranges(g, p, which), u, b, y, sc, cga);
}

// p_new = r + beta p_old on the boundary planes facing a neighbour (they are
// the neighbours' halos, sent before phase A): the gather path's map
// arithmetic, no x update (phase A does it for every own node); card
// components (sparse fields: component stride sp.cs)
__global__ void k_sp_pmap(double *pn, const double *po, const double *r, int64_t cs, int card, int64_t a0,
                          int64_t n0, int64_t a1, int64_t n1, const CgScal *sc) {
    if (sc->status != 0) return;
    const double beta = sc->beta;
    const int64_t n = n0 + n1;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < card * n; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = t / n, k = t % n;
        const int64_t i = c * cs + (k < n0 ? a0 + k : a1 + (k - n0));
        pn[i] = fma(beta, po[i], r[i]);
    }
}

nb_status nb_sparse_pmap(nb_grid *g, int p, int card, const double *po, const double *r, double *pn,
                         const CgScal *sc) {
    const NbPart &q = g->parts[p];
    const NbSparsePart &sp = g->sp[p];
    const int nz = q.nz();
    int64_t a0 = 0, n0 = 0, a1 = 0, n1 = 0;
    if (q.lo >= 0) a0 = sp.hl + sp.pstart[0], n0 = sp.pstart[1] - sp.pstart[0];
    if (q.hi >= 0 && (q.lo < 0 || nz > 1)) a1 = sp.hl + sp.pstart[nz - 1], n1 = sp.pstart[nz] - sp.pstart[nz - 1];
    if (n0 + n1 <= 0) return NB_OK;
    LaunchScope ls(g, g->cs, "k_sp_cg_map");
    k_sp_pmap<<<(unsigned)std::min<int64_t>((card * (n0 + n1) + 255) / 256, 148 * 8), 256, 0, g->cs>>>(
        pn, po, r, sp.cs, card, a0, n0, a1, n1, sc);
    return nb_launch_check("k_sp_pmap");
}

// build the tables and every list the CG / apply use (outside any capture)
nb_status nb_sparse_fem_box_prepare(nb_grid *g) {
    NB_TRY(nb_sparse_fem_box_tables(g));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p)
        for (int which = 0; which < 3; ++which) {
            const int4 *it;
            int64_t n;
            NB_TRY(nb_sparse_fem_box_list(g, p, sp_box_ranges(g, p, which), NB_SFB_ZC, &it, &n, false));
            NB_TRY(nb_sparse_fem_box_list(g, p, sp_box_ranges(g, p, which), NB_SFB_ZC, &it, &n, true));
            NB_TRY(nb_sparse_fem_box_list(g, p, sp_box_ranges(g, p, which), NB_SFB_ZC, &it, &n, false, 16));
        }
    return nb_sparse_tile_tp(g);
}

nb_status nb_sparse_fem_rhs(nb_field *b, double pr);

static nb_status fem_check(const nb_field *u) {
    if (!u) NB_FAIL(NB_EINVAL, "NULL field");
    if (u->dt != NB_F64 || u->card != 3) NB_FAIL(NB_EMISMATCH, "FEM fields are fp64 with cardinality 3");
    NB_LAYOUTS(u, (1 << NB_SOA) | (1 << NB_SOA_PLANE), "FEM");
    return NB_OK;
}

extern "C" nb_status nb_fem27_apply(const nb_field *u, nb_field *y, double E, double nu) {
    NB_TRY(fem_check(u));
    NB_TRY(fem_check(y));
    if (u->g != y->g) NB_FAIL(NB_EMISMATCH, "fields belong to different grids");
    nb_grid *g = u->g;
    cudaSetDevice(g->device);
    NB_TRY(fem_upload_constants(E, nu));
    if (g->sparse) {
        const bool box = nb_sparse_fem_boxed();
        NB_TRY(box ? nb_sparse_fem_box_prepare(g) : nb_sparse_fem_tables(g, true));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            const NbSparsePart &sp = g->sp[p];
            if (box)
                NB_TRY(nb_sparse_fem_box_ranges(g, p, 0, (const double *)u->base[p], nullptr, (double *)y->base[p],
                                                nullptr, 0, nullptr));
            else
                NB_TRY(nb_sparse_fem_pass(g, p, 0, sp.d_seg, nullptr, 0, sp.seg_start.back(),
                                          (const double *)u->base[p], nullptr, (double *)y->base[p], nullptr));
        }
        return NB_OK;
    }
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
    if (g->sparse) return nb_sparse_fem_rhs(b, pressure);
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
    if (g->sparse) {
        const bool box = nb_sparse_fem_boxed();
        NB_TRY(nb_sparse_fem_tables(g, !box));  // the gather pass needs the row bases
        if (box) NB_TRY(nb_sparse_fem_box_prepare(g));  // the q pass's lists, before any capture
        // fused phase A (p ping-pong) with NB_SPF_FUSED=1, decided once per
        // solver: same bits, but 2.70 ms against 1.24 + 1.00 ms for the box
        // q pass after the separate map at 384^3 — its 8-byte cp.async
        // staging of six arrays per plane leaves it waiting on data (ncu:
        // 39 % issue, half the stall samples at the ring wait and barrier)
        cg->pingpong = box && getenv("NB_SPF_FUSED");
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            const NbSparsePart &sp = g->sp[p];
            double *r = (double *)cg->r->base[p];
            if (box) {
                NB_TRY(nb_sparse_fem_box_ranges(g, p, 0, (const double *)cg->x->base[p],
                                                (const double *)cg->b->base[p], r, nullptr, 2, nullptr));
                NB_TRY(nb_sparse_fem_dot(g, p, r, r, nullptr));
            } else {
                NB_TRY(nb_sparse_fem_pass(g, p, 2, sp.d_seg, nullptr, 0, sp.seg_start.back(),
                                          (const double *)cg->x->base[p], (const double *)cg->b->base[p], r, nullptr));
            }
        }
        return nb_reduce_finalize(g, 3, FIN_CG_INIT, cg->sc, 0);
    }
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        FemArgs A{};
        A.u = (const double *)cg->x->base[p];
        A.b = (const double *)cg->b->base[p];
        A.y = (double *)cg->r->base[p];
        NB_TRY(fem_launch<FEM_CG_INIT>(g, p, A, cg->x, 0, g->parts[p].nz(), "k_fem_cg_init"));
    }
    return nb_reduce_finalize(g, 3, FIN_CG_INIT, cg->sc, 0);
}

// fused schedule (default): boundary planes of p_new -> halo(p_new) ->
// surface nodes + fused phase A -> alpha -> r -= alpha q, <r,r> -> beta
// (216 B/node/iter).  With NB_FEM_KERNEL (reference kernels) or NB_FEM_3PASS:
// map -> halo(p_new) -> q = K p_new -> alpha -> r -> beta (240 B/node/iter).
// Both compute the same values in the same order (bitwise).
static bool fem_fused() { return !getenv("NB_FEM_KERNEL") && !getenv("NB_FEM_3PASS") && nb_tma_enabled(); }

nb_status nb_sparse_fem_cg_hooks(nb_cg *cg, int parity);  // nb_sparse.cu

nb_status nb_fem_cg_hooks(nb_cg *cg, int parity) {
    nb_grid *g = cg->g;
    if (g->sparse) return nb_sparse_fem_cg_hooks(cg, parity);
    nb_field *pn = cg->p[parity], *po = cg->p[parity ^ 1];
    const bool fused = fem_fused();
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbPart &q = g->parts[p];
        // fused: only the boundary planes (the neighbours' halos; phase A
        // forms p_new everywhere else), all planes x components in ONE launch
        FemMapSegs S{};
        int nseg = 0;
        int64_t n = 0;
        if (fused) {
            n = pn->plane;  // one component's plane (SOA and SOA_PLANE)
            for (int c = 0; c < 3; ++c) {
                if (q.lo >= 0) S.off[nseg++] = (int64_t)c * fcs(pn, p) + pn->ps;
                if (q.hi >= 0 && q.nz() > 1) S.off[nseg++] = (int64_t)c * fcs(pn, p) + (int64_t)q.nz() * pn->ps;
            }
        } else if (pn->layout == NB_SOA_PLANE) {  // all own planes of all components: one range
            n = (int64_t)q.nz() * pn->ps;
            S.off[nseg++] = pn->ps;
        } else {
            n = (int64_t)q.nz() * pn->ps;
            for (int c = 0; c < 3; ++c) S.off[nseg++] = (int64_t)c * fcs(pn, p) + pn->ps;
        }
        if (!nseg) continue;
        LaunchScope ls(g, g->cs, "k_fem_map");
        k_fem_map<<<dim3(fused ? 148 : 148 * 8, nseg), 256, 0, g->cs>>>(
            (double *)cg->x->base[p], (double *)pn->base[p], (const double *)po->base[p], (const double *)cg->r->base[p],
            S, n, cg->sc, fused ? 0 : 1);
        NB_TRY(nb_launch_check("k_fem_map"));
    }
    // OCC (occ != NONE, fused schedule, and a transfer
    // that actually runs asynchronously: the peer or NCCL transport across
    // processes, or NB_HALO_STREAM): the halo of p_new is sent right after
    // the boundary-plane map, and the surface nodes of the planes whose
    // neighbours are own planes ([lo, nz - hi)) are computed while it is in
    // flight (they recompute p_new at their neighbours from r and p_old);
    // after the wait the surface nodes of the boundary planes, then the
    // streaming phase A over all planes in one launch.  Same values, same
    // order per node and per-plane dot partials: bitwise equal to the serial
    // schedule.  In one process with fused halos the copies are stream-
    // ordered work with nothing to overlap, and the serial schedule runs.
    const bool split = fused && cg->prm.occ != NB_OCC_NONE && g->nparts > 1 &&
                       (nb_is_peer(g) || nb_halo_on_stream(g)) && nb_tma_enabled() && !getenv("NB_FEM_KERNEL");
    auto args = [&](int p) {
        FemArgs A{};
        A.y = (double *)cg->q->base[p];
        A.sc = cg->sc;
        if (fused) {
            A.r = (const double *)cg->r->base[p];
            A.po = (const double *)po->base[p];
            A.pn = (double *)pn->base[p];
            A.x = (double *)cg->x->base[p];
        } else {
            A.u = (const double *)pn->base[p];
        }
        return A;
    };
    if (!split) {
        NB_TRY(nb_halo_exchange_planes(pn, 0, 3, true, true, g->cs));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            if (fused)
                NB_TRY(fem_launch<FEM_CG_A>(g, p, args(p), pn, 0, g->parts[p].nz(), "k_fem_cg_a"));
            else
                NB_TRY(fem_launch<FEM_CG_Q>(g, p, args(p), pn, 0, g->parts[p].nz(), "k_fem_cg_q"));
        }
    } else {
        NB_TRY(nb_halo_split_begin(pn, 0, 3, cg->hs));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            const NbPart &q = g->parts[p];
            const int ib = q.lo >= 0 ? 1 : 0, ie = q.nz() - (q.hi >= 0 ? 1 : 0);
            if (ie > ib) NB_TRY(fem_launch<FEM_CG_A>(g, p, args(p), pn, ib, ie, "k_fem_cg_a", FEM_SURF));
        }
        NB_TRY(nb_halo_split_wait(g, cg->hs));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            const NbPart &q = g->parts[p];
            // the surface nodes of both boundary planes in one launch per kernel
            if (q.lo >= 0 && q.hi >= 0 && q.nz() > 1)
                NB_TRY(fem_launch<FEM_CG_A>(g, p, args(p), pn, 0, 1, "k_fem_cg_a", FEM_SURF, q.nz() - 1));
            else if (q.lo >= 0)
                NB_TRY(fem_launch<FEM_CG_A>(g, p, args(p), pn, 0, 1, "k_fem_cg_a", FEM_SURF));
            else if (q.hi >= 0)
                NB_TRY(fem_launch<FEM_CG_A>(g, p, args(p), pn, q.nz() - 1, q.nz(), "k_fem_cg_a", FEM_SURF));
            NB_TRY(fem_launch<FEM_CG_A>(g, p, args(p), pn, 0, q.nz(), "k_fem_cg_a", FEM_BULK));
        }
    }
    NB_TRY(nb_reduce_finalize(g, 3, FIN_CG_PQ, cg->sc, 0));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        PGeo geo = pgeo(pn, p);
        LaunchScope ls(g, g->cs, "k_fem_r");
        if (getenv("NB_FEM_R_PLANE")) {  // one CTA per tile and plane (the earlier kernel)
            dim3 blk(DOT_TX, DOT_TY), grd(g->tiles_x, g->tiles_y, geo.nzl);
            k_fem_r<<<grd, blk, 0, g->cs>>>((double *)cg->r->base[p], (const double *)cg->q->base[p], fcs(pn, p), geo,
                                            0, cg->sc, g->tp, g->T);
        } else {
            dim3 blk(DOT_TX, DOT_TY), grd(g->tiles_x, g->tiles_y, (geo.nzl + FRZ - 1) / FRZ);
            k_fem_rz<<<grd, blk, 0, g->cs>>>((double *)cg->r->base[p], (const double *)cg->q->base[p], fcs(pn, p), geo,
                                             0, geo.nzl, cg->sc, g->tp, g->T);
        }
        NB_TRY(nb_launch_check("k_fem_r"));
    }
    NB_TRY(nb_reduce_finalize(g, 3, FIN_CG_RR, cg->sc, 0));
    cg->k += 1;
    return NB_OK;
}
