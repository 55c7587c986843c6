// nb_stencil.cu — 7-point stencil, the config-C1 map-stencil-reduce loop and
// the matrix-free Poisson CG on dense grids.
//
// Paper: Listing 2 7-point Laplacian, Fig. 4a chain
// apxpy -> laplace -> dot (L268-L280), CG with UpdateP first (L161-L163,
// L460), OCC variants (L293-L331).  DESIGN.md "Kernels" gives the roofline of
// every kernel; "CG schedule" the 64 B/cell/iteration two-phase schedule.
//
// Per-cell arithmetic is fixed:
//   s = ((((x[-x] + x[+x]) + x[-y]) + x[+y]) + x[-z]) + x[+z]
//   L(x) = fma(-6, x_c, s)          A(p) = -L(p) = fma(6, p_c, -s)
//   UpdateP: p = fma(beta, p_old, r)   x-update: x = fma(alpha, p, x)
//   r-update: r = fma(-alpha, q, r)    C1 map: x = fma(a, y, x)
// Every kernel that touches a cell runs these same expressions, so the
// result does not depend on the partition count or the OCC schedule.
#include <algorithm>
#include <map>
#include <vector>

#include "nb_device.cuh"
#include "nb_internal.cuh"
#include "nb_zmarch.cuh"

#ifndef NB_ZL_SMEM
#define NB_ZL_SMEM 1
#endif
#ifndef NB_ZL_L1
#define NB_ZL_L1 0
#endif

std::vector<std::pair<int, int>> view_ranges(const nb_grid *g, int p, nb_view v);
nb_status nb_dot_partials(const nb_field *x, const nb_field *y);
nb_status nb_sparse_laplace7(const nb_field *x, nb_field *y, nb_view v);
bool nb_tma_enabled();
nb_status nb_cgB_tma(nb_grid *g, const PGeo &geo, const double *p, double *r, int zb, int ze, const CgScal *sc);
nb_status nb_c1_tma(nb_grid *g, const PGeo &geo, const double *xin, const double *yin, double *xout, double *yout,
                    double a, bool domap, int zb, int ze, int zhi = -1);
nb_status nb_c1_finalize_all(nb_grid *g, int iters);
nb_status nb_cgA_tma(nb_grid *g, const PGeo &geo, const double *r, const double *po, double *pn, double *x, bool domap,
                     int zb, int ze, const CgScal *sc, int zhi = -1);

static inline int64_t dcs(const nb_field *f, int p) { return nb_cstride(f, p); }


// ===========================================================================
// 7-point Laplacian y = L(x) (Listing 2).  Algorithmic traffic: read x +
// write y = 2*sizeof(T) per cell.
// ===========================================================================
// NEG: y = -L(x) = fma(6, x_c, -s), the CG operator A (bitwise the CG's A p)
template <typename TT, bool NEG = false>
struct Lap7Op {
    using T = TT;
    struct Raw {
        TT a;
    };
    static constexpr bool DOT = false, MAP = false;
    const TT *x;
    TT *y;
    TT outv;
    __device__ bool skip() const { return false; }
    __device__ void init() {}
    __device__ TT outside() const { return outv; }
    __device__ Raw raw(int, int64_t i, bool) const { return {x[i]}; }
    __device__ TT val(int, const Raw &r) const { return r.a; }
    __device__ TT nval(int, int64_t i) const { return x[i]; }
    __device__ double cell(int, int64_t i, TT c, TT s, const Raw &) {
        __stcs(y + i, NEG ? fma(TT(6), c, -s) : fma(TT(-6), c, s));
        return 0.0;
    }
};

template <class Op, bool SMEM = false>
static nb_status launch_zmarch(nb_grid *g, const char *name, Op op, PGeo geo, int zb, int ze) {
    if (ze <= zb) return NB_OK;
    constexpr int ZR = Op::MAP ? ZR_MAP : ZR_STO;
    constexpr int ZTY = ZW * ZR;
    dim3 blk(32 * ZW), grd(g->tiles_x, (g->ny + ZTY - 1) / ZTY, (ze - zb + ZC - 1) / ZC);
    LaunchScope ls(g, g->cs, name);
    constexpr int L = SMEM ? NB_ZL_SMEM : NB_ZL_L1;
    k_zmarch<Op, SMEM, L, ZR><<<grd, blk, 0, g->cs>>>(op, geo, zb, ze, g->tp, g->T, g->tiles_y);
    return nb_launch_check(name);
}

extern "C" nb_status nb_laplace7(const nb_field *x, nb_field *y, nb_view v) {
    return nb_stencil7(x, y, v, false);
}

// y = L(x) (neg = false) or y = A x = -L(x) (neg = true) on the view
nb_status nb_stencil7(const nb_field *x, nb_field *y, nb_view v, bool neg) {
    if (!x || !y) NB_FAIL(NB_EINVAL, "nb_laplace7: NULL field");
    if (x->g != y->g) NB_FAIL(NB_EMISMATCH, "fields belong to different grids");
    if (x->dt != y->dt || x->card != 1 || y->card != 1)
        NB_FAIL(NB_EMISMATCH, "nb_laplace7 needs two scalar fields of one dtype");
    nb_grid *g = x->g;
    if (g->sparse) {
        if (neg) NB_FAIL(NB_EUNSUPPORTED, "-L on element-sparse grids");
        return nb_sparse_laplace7(x, y, v);
    }
    cudaSetDevice(g->device);
    for (int p = 0; p < g->nparts; ++p) {
        if (!g->parts[p].local) continue;
        PGeo geo = pgeo(x, p);
        for (auto rg : view_ranges(g, p, v)) {
            const double *xd = (const double *)x->base[p];
            double *yd = (double *)y->base[p];
            const float *xf = (const float *)x->base[p];
            float *yf = (float *)y->base[p];
            if (x->dt == NB_F64 && !neg)
                NB_TRY(launch_zmarch(g, "k_laplace7", Lap7Op<double>{xd, yd, x->outside}, geo, rg.first, rg.second));
            else if (x->dt == NB_F64)
                NB_TRY(launch_zmarch(g, "k_laplace7", Lap7Op<double, true>{xd, yd, x->outside}, geo, rg.first,
                                     rg.second));
            else if (!neg)
                NB_TRY(launch_zmarch(g, "k_laplace7", Lap7Op<float>{xf, yf, (float)x->outside}, geo, rg.first,
                                     rg.second));
            else
                NB_TRY(launch_zmarch(g, "k_laplace7", Lap7Op<float, true>{xf, yf, (float)x->outside}, geo, rg.first,
                                     rg.second));
        }
    }
    return NB_OK;
}

// ===========================================================================
// "map then stencil then reduce" fused z-march (the Fig. 4a chain and CG
// phase A share it).  The map output u = fma(m, v, w) is recomputed at every
// neighbour inside the partition (never read back from memory), and read
// from the stored u buffer on halo planes, where it was written by the
// neighbour's boundary map.  MODE:
//   MSR_C1: u = x_new = fma(a, y, x); out = y_new = L(u); dot = u*out
//   MSR_CG: u = p_new = fma(beta, p_old, r); out = q = A(u); dot = u*q; also
//           applies the deferred x += alpha_prev * p_old when DOMAP
// ===========================================================================
enum { MSR_C1 = 0, MSR_CG = 1 };

struct MsrArgs {
    const double *w;   // C1: x_in ; CG: r
    const double *v;   // C1: y_in ; CG: p_old
    double *u;         // C1: x_out ; CG: p_new   (halo planes read from here)
    double *out;       // C1: y_out ; CG: unused
    double *xs;        // CG: solution x (deferred update) ; C1: unused
    double m;          // C1: a ; CG: beta
    double ap;         // CG: alpha_prev
    int pending;       // CG: apply deferred x update
    const CgScal *sc;  // CG: status gate (may be NULL)
};

template <int MODE, bool RECOMPUTE, bool DOMAP>
struct MsrOp {
    using T = double;
    struct Raw {
        double v, w, x;  // v: map input (or stored u on halo planes), w, x: see cell()
    };
    static constexpr bool DOT = true, MAP = true;  // every MsrOp variant: one canonical <u, res> order
    MsrArgs A;
    int nzl;
    double m, ap;
    int pending;
    __device__ bool skip() const { return A.sc && A.sc->status != 0; }
    __device__ void init() {
        m = A.m;
        ap = A.ap;
        pending = A.pending;
        if (MODE == MSR_CG) {  // beta, alpha_prev, pending live on the device
            m = A.sc->beta;
            ap = A.sc->alpha_prev;
            pending = A.sc->pending;
        }
    }
    __device__ double outside() const { return 0.0; }
    __device__ bool stored(int zl) const { return !RECOMPUTE || zl < 0 || zl >= nzl; }
    // map output: recomputed inside the slab, read back on halo planes
    __device__ Raw raw(int zl, int64_t i, bool own) const {
        Raw r{0.0, 0.0, 0.0};
        if (stored(zl)) {
            r.v = A.u[i];
        } else {
            r.v = A.v[i];
            r.w = A.w[i];
            if (MODE == MSR_CG && DOMAP && own && pending) r.x = A.xs[i];
        }
        return r;
    }
    __device__ double val(int zl, const Raw &r) const { return stored(zl) ? r.v : fma(m, r.v, r.w); }
    __device__ double nval(int zl, int64_t i) const { return val(zl, raw(zl, i, false)); }
    __device__ double cell(int, int64_t i, double c, double s, const Raw &rc) {
        double res;
        if (MODE == MSR_C1) {
            res = fma(-6.0, c, s);
            __stcs(A.out + i, res);
        } else {
            res = fma(6.0, c, -s);
        }
        if (DOMAP) {
            A.u[i] = c;
            if (MODE == MSR_CG && pending) A.xs[i] = fma(ap, rc.v, rc.x);
        }
        return __dmul_rn(c, res);
    }
};

// ===========================================================================
// Specialised recompute kernel (the CG phase-A / C1 hot path): the same
// arithmetic and canonical dot order as k_zmarch<MsrOp<MODE, true, DOMAP>,
// SMEM, L=1, ZR=1>, written with per-array pointers advanced by one plane per
// step, a CTA-uniform fast path for tiles whose cells and ring are all inside
// the domain, and halo-plane selection by CTA-uniform branches — about a
// third of the generic kernel's instructions per cell.
// ===========================================================================
template <int MODE, bool DOMAP, bool FULL>
__device__ __forceinline__ void msr_fast_body(const MsrArgs &A, const PGeo &g, int zs, int zend, double m, double ap,
                                              bool dox, double (*sU)[DOT_TY + 2][DOT_TX + 2], double (*sw)[ZW]) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int x0 = blockIdx.x * DOT_TX, y0 = blockIdx.y * DOT_TY;
    const int xi = x0 + lane, yi = y0 + w;
    const int nzl = g.nzl;
    const int64_t ps = g.ps;
    const bool valid = FULL || (xi < g.nx && yi < g.ny);
    // ring roles: warp 0 / 7 -> rows y0-1 / y0+8, lane 0 / 31 -> columns x0-1 / x0+32
    const bool hasR = (w == 0 || w == DOT_TY - 1), hasC = (lane == 0 || lane == 31);
    const int ry = w == 0 ? y0 - 1 : y0 + DOT_TY, rx = lane == 0 ? x0 - 1 : x0 + DOT_TX;
    const bool rin = hasR && (FULL || (xi < g.nx && ry >= 0 && ry < g.ny));
    const bool cin = hasC && (FULL || (rx >= 0 && rx < g.nx && yi < g.ny));
    // element offsets of plane zs-1 (halo or in-slab), advanced by ps per step
    int64_t eo = valid ? (int64_t)zs * ps + (int64_t)yi * g.pitch + xi : 0;
    int64_t er = rin ? (int64_t)(zs + 1) * ps + (int64_t)ry * g.pitch + xi : 0;
    int64_t ec = cin ? (int64_t)(zs + 1) * ps + (int64_t)yi * g.pitch + rx : 0;
    auto U = [&](int zl, int64_t e) -> double {  // map output at plane zl (uniform halo test)
        return (zl < 0 || zl >= nzl) ? A.u[e] : fma(m, A.v[e], A.w[e]);
    };
    double below = 0.0, center = 0.0, vc = 0.0, xc = 0.0;
    // raw loads of plane zs+1 (own and ring) and of plane zs (ring)
    double va = 0.0, wa = 0.0, xa = 0.0, rv = 0.0, rw = 0.0, cv = 0.0, cw = 0.0;
    if (valid) {
        below = U(zs - 1, eo);
        eo += ps;  // plane zs
        vc = A.v[eo];
        center = fma(m, vc, A.w[eo]);
        if (dox) xc = A.xs[eo];
        if (zs + 1 < nzl) {
            va = A.v[eo + ps];
            wa = A.w[eo + ps];
            if (dox) xa = A.xs[eo + ps];
        } else {
            va = A.u[eo + ps];
        }
    }
    sU[0][w + 1][lane + 1] = center;
    if (hasR) sU[0][w == 0 ? 0 : DOT_TY + 1][lane + 1] = rin ? fma(m, A.v[er], A.w[er]) : 0.0;
    if (hasC) sU[0][w + 1][lane == 0 ? 0 : DOT_TX + 1] = cin ? fma(m, A.v[ec], A.w[ec]) : 0.0;
    if (zs + 1 < zend) {
        if (rin) { rv = A.v[er + ps]; rw = A.w[er + ps]; }
        if (cin) { cv = A.v[ec + ps]; cw = A.w[ec + ps]; }
    }
#pragma unroll 2
    for (int z = zs; z < zend; ++z) {
        const int b = (z - zs) & 1;
        // prefetch plane z+2 (own) and the ring of plane z+2
        double vb = 0.0, wb = 0.0, xb = 0.0, rvb = 0.0, rwb = 0.0, cvb = 0.0, cwb = 0.0;
        if (z + 2 <= zend) {
            if (z + 2 < nzl) {
                if (valid) {
                    vb = A.v[eo + 2 * ps];
                    wb = A.w[eo + 2 * ps];
                    if (dox) xb = A.xs[eo + 2 * ps];
                }
            } else if (valid) {
                vb = A.u[eo + 2 * ps];
            }
        }
        if (z + 2 < zend) {
            if (rin) { rvb = A.v[er + 2 * ps]; rwb = A.w[er + 2 * ps]; }
            if (cin) { cvb = A.v[ec + 2 * ps]; cwb = A.w[ec + 2 * ps]; }
        }
        const double above = (z + 1 < nzl) ? fma(m, va, wa) : va;
        __syncthreads();
        double prod = 0.0;
        if (valid) {
            double s = __dadd_rn(sU[b][w + 1][lane], sU[b][w + 1][lane + 2]);
            s = __dadd_rn(s, sU[b][w][lane + 1]);
            s = __dadd_rn(s, sU[b][w + 2][lane + 1]);
            s = __dadd_rn(s, below);
            s = __dadd_rn(s, above);
            double res;
            if (MODE == MSR_C1) {
                res = fma(-6.0, center, s);
                __stcs(A.out + eo, res);
            } else {
                res = fma(6.0, center, -s);
            }
            if (DOMAP) {
                A.u[eo] = center;
                if (dox) A.xs[eo] = fma(ap, vc, xc);
            }
            prod = __dmul_rn(center, res);
        }
        prod = warp_sum_canon(prod);
        if (lane == 0) sw[z - zs][w] = prod;
        if (z + 1 < zend) {
            sU[b ^ 1][w + 1][lane + 1] = above;
            if (hasR) sU[b ^ 1][w == 0 ? 0 : DOT_TY + 1][lane + 1] = rin ? fma(m, rv, rw) : 0.0;
            if (hasC) sU[b ^ 1][w + 1][lane == 0 ? 0 : DOT_TX + 1] = cin ? fma(m, cv, cw) : 0.0;
        }
        below = center;
        center = above;
        vc = va;
        xc = xa;
        va = vb;
        wa = wb;
        xa = xb;
        rv = rvb;
        rw = rwb;
        cv = cvb;
        cw = cwb;
        eo += ps;
        er += ps;
        ec += ps;
    }
}

template <int MODE, bool DOMAP>
__global__ void __launch_bounds__(DOT_TX *DOT_TY) k_msr_fast(MsrArgs A, PGeo g, int zb, int ze, double *tp, int T,
                                                           int tiles_y, int zc) {
    __shared__ double sU[2][DOT_TY + 2][DOT_TX + 2];
    __shared__ double sw[ZC][ZW];
    if (A.sc && A.sc->status != 0) return;
    double m = A.m, ap = A.ap;
    int pending = A.pending;
    if (MODE == MSR_CG) {
        m = A.sc->beta;
        ap = A.sc->alpha_prev;
        pending = A.sc->pending;
    }
    const bool dox = MODE == MSR_CG && DOMAP && pending;
    const int zs = zb + blockIdx.z * zc, zend = min(ze, zs + zc);  // zc <= ZC planes per CTA
    const int x0 = blockIdx.x * DOT_TX, y0 = blockIdx.y * DOT_TY;
    // all own cells and all ring cells inside the domain (CTA-uniform)
    const bool full = x0 >= 1 && y0 >= 1 && x0 + DOT_TX + 1 <= g.nx && y0 + DOT_TY + 1 <= g.ny;
    if (full)
        msr_fast_body<MODE, DOMAP, true>(A, g, zs, zend, m, ap, dox, sU, sw);
    else
        msr_fast_body<MODE, DOMAP, false>(A, g, zs, zend, m, ap, dox, sU, sw);
    __syncthreads();
    zm_flush<1>(sw, zend - zs, tp, (int64_t)g.z0 + zs, T, gridDim.x, tiles_y, blockIdx.x, blockIdx.y);
}

// map only: u = fma(m, v, w) on planes [zb, ze) (+ CG deferred x update);
// boundary planes are also stored into the neighbour partition's halo plane
// (rem_lo: lower neighbour's high halo, rem_hi: upper neighbour's low halo)
// — the halo transfer fused into the producing kernel.
template <int MODE>
// planes [zb, ze), or with zhi >= 0 the pair {zb, zhi} (one per blockIdx.z):
// both boundary planes of a slab in one launch
__global__ void __launch_bounds__(256) k_map_u(MsrArgs A, PGeo g, int zb, int ze, int zhi, double *rem_lo,
                                               double *rem_hi) {
    if (A.sc && A.sc->status != 0) return;
    double m = A.m, ap = A.ap;
    int pending = A.pending;
    if (MODE == MSR_CG) {
        m = A.sc->beta;
        ap = A.sc->alpha_prev;
        pending = A.sc->pending;
    }
    const int xi = blockIdx.x * blockDim.x + threadIdx.x, yi = blockIdx.y;
    if (xi >= g.nx) return;
    if (zhi >= 0) {
        zb = blockIdx.z ? zhi : zb;
        ze = zb + 1;
    }
    for (int z = zb + (zhi >= 0 ? 0 : (int)blockIdx.z); z < ze; z += gridDim.z) {
        const int64_t row = (int64_t)yi * g.pitch + xi;
        const int64_t ic = row + (int64_t)(z + 1) * g.ps;
        double vc = A.v[ic];
        double u = fma(m, vc, A.w[ic]);
        A.u[ic] = u;
        if (z == 0 && rem_lo) rem_lo[row] = u;
        if (z == g.nzl - 1 && rem_hi) rem_hi[row] = u;
        if (MODE == MSR_CG && pending) A.xs[ic] = fma(ap, vc, A.xs[ic]);
    }
}

// CG phase B: q = A(p_new) from stored p_new (halo planes included),
// r = fma(-alpha, q, r), dot r*r.
struct CgBOp {
    using T = double;
    struct Raw {
        double p, r;
    };
    static constexpr bool DOT = true, MAP = false;
    const double *p;
    double *r;
    const CgScal *sc;
    double alpha;
    __device__ bool skip() const { return sc->status != 0; }
    __device__ void init() { alpha = sc->alpha; }
    __device__ double outside() const { return 0.0; }
    __device__ Raw raw(int, int64_t i, bool own) const { return {p[i], own ? __ldcs(r + i) : 0.0}; }
    __device__ double val(int, const Raw &q) const { return q.p; }
    __device__ double nval(int, int64_t i) const { return p[i]; }
    __device__ double cell(int, int64_t i, double c, double s, const Raw &rc) {
        double q = fma(6.0, c, -s);
        double rn = fma(-alpha, q, rc.r);
        __stcs(r + i, rn);
        return __dmul_rn(rn, rn);
    }
};

// CG set-up: r = b - A(x) (x halo current), dot r*r
struct CgInitOp {
    using T = double;
    struct Raw {
        double x, b;
    };
    static constexpr bool DOT = true, MAP = false;
    const double *x, *b;
    double *r;
    double outv;
    __device__ bool skip() const { return false; }
    __device__ void init() {}
    __device__ double outside() const { return outv; }
    __device__ Raw raw(int, int64_t i, bool own) const { return {x[i], own ? b[i] : 0.0}; }
    __device__ double val(int, const Raw &q) const { return q.x; }
    __device__ double nval(int, int64_t i) const { return x[i]; }
    __device__ double cell(int, int64_t i, double c, double s, const Raw &rc) {
        double ax = fma(6.0, c, -s);
        double rv = __dsub_rn(rc.b, ax);
        r[i] = rv;
        return __dmul_rn(rv, rv);
    }
};

// x += alpha_prev * p_last if an update is pending (p_last chosen by the
// device iteration count, since convergence may stop the count early)
__global__ void __launch_bounds__(256) k_cg_flush(double *x, const double *p0, const double *p1, int64_t n,
                                                  CgScal *sc) {
    if (!sc->pending) return;
    const double *p = (sc->iters & 1) ? p1 : p0;
    const double a = sc->alpha_prev;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[i] = fma(a, p[i], x[i]);
}

__global__ void k_cg_flush_done(CgScal *sc) {
    if (threadIdx.x == 0 && blockIdx.x == 0) sc->pending = 0;
}

// ===========================================================================
// schedules
// ===========================================================================
// Boundary-plane ranges of partition p that face another partition.
static std::vector<int> bnd_planes(const nb_grid *g, int p) {
    std::vector<int> r;
    const NbPart &q = g->parts[p];
    if (q.lo >= 0) r.push_back(0);
    if (q.hi >= 0 && !(q.lo >= 0 && q.nz() == 1)) r.push_back(q.nz() - 1);
    return r;
}

// pointer to plane zl of partition p of a scalar field
static double *pl(const nb_field *f, int p, int zl) {
    return (double *)f->base[p] + (int64_t)(zl + 1) * f->ps;
}

// launch k_map_u on the planes of `planes` (or all when all==true), with
// fused stores into neighbour halos of `ufield` for local neighbours
static nb_status launch_map_u(nb_grid *g, int mode, int p, MsrArgs A, const nb_field *ufield, int zb, int ze,
                              int zhi = -1) {
    const NbPart &q = g->parts[p];
    PGeo geo = pgeo(ufield, p);
    double *rem_lo = nullptr, *rem_hi = nullptr;
    if (!nb_halo_on_stream(g)) {  // fused halo: store straight into the neighbour
        if (zb == 0 && nb_reachable(ufield, q.lo)) rem_lo = pl(ufield, q.lo, g->parts[q.lo].nz());
        if ((ze == q.nz() || zhi == q.nz() - 1) && nb_reachable(ufield, q.hi)) rem_hi = pl(ufield, q.hi, -1);
    }
    dim3 blk(128), grd((g->nx + 127) / 128, g->ny, zhi >= 0 ? 2 : std::min(ze - zb, 64));
    LaunchScope ls(g, g->cs, "k_map_u");
    if (mode == MSR_C1)
        k_map_u<MSR_C1><<<grd, blk, 0, g->cs>>>(A, geo, zb, ze, zhi, rem_lo, rem_hi);
    else
        k_map_u<MSR_CG><<<grd, blk, 0, g->cs>>>(A, geo, zb, ze, zhi, rem_lo, rem_hi);
    return nb_launch_check("k_map_u");
}

// the boundary planes of partition p as one (zb, zhi) launch pair when there
// are two (zhi = -1: a single plane zb)
static std::pair<int, int> bnd_pair(const nb_grid *g, int p) {
    auto b = bnd_planes(g, p);
    if (b.empty()) return {-1, -1};
    if (b.size() == 1) return {b[0], -1};
    return {b[0], b[1]};
}

template <int MODE, bool RC, bool DM>
static nb_status launch_msr(nb_grid *g, int p, MsrArgs A, const nb_field *f, int zb, int ze, int zhi = -1) {
    if (ze <= zb) return NB_OK;
    const char *name = MODE == MSR_C1 ? "k_msr_c1" : "k_msr_cgA";
    if (MODE == MSR_CG && RC && ZR_MAP == 1 && nb_tma_enabled())  // TMA-staged phase A
        return nb_cgA_tma(g, pgeo(f, p), A.w, A.v, A.u, A.xs, DM, zb, ze, A.sc, zhi);
    // TMA-staged C1 chain: large grids only (the 64^3 C1 config lives in L2,
    // where the register/L1 kernel has lower latency per launch)
    if (MODE == MSR_C1 && RC && ZR_MAP == 1 && nb_tma_enabled() && (int64_t)g->nx * g->ny * g->nz >= (1 << 21))
        return nb_c1_tma(g, pgeo(f, p), A.w, A.v, A.u, A.out, A.m, DM, zb, ze, zhi);
    if (zhi >= 0) {  // the other kernels take plane ranges: the pair as two launches
        NB_TRY((launch_msr<MODE, RC, DM>(g, p, A, f, zb, ze)));
        return launch_msr<MODE, RC, DM>(g, p, A, f, zhi, zhi + 1);
    }
    if (RC && ZR_MAP == 1 && !getenv("NB_GENERIC_MSR")) {
        // specialised recompute kernel (same arithmetic and dot order); planes
        // per CTA halved while the launch has fewer than two CTAs per SM (the
        // dot partials are per plane and tile: results do not depend on it)
        int zc = ZC;
        while (zc > 2 && (int64_t)g->tiles_x * g->tiles_y * ((ze - zb + zc - 1) / zc) < 2 * 148) zc /= 2;
        dim3 blk(DOT_TX * DOT_TY), grd(g->tiles_x, g->tiles_y, (ze - zb + zc - 1) / zc);
        LaunchScope ls(g, g->cs, name);
        k_msr_fast<MODE, DM><<<grd, blk, 0, g->cs>>>(A, pgeo(f, p), zb, ze, g->tp, g->T, g->tiles_y, zc);
        return nb_launch_check(name);
    }
    MsrOp<MODE, RC, DM> op;
    op.A = A;
    op.nzl = g->parts[p].nz();
    // recompute: the map output of every cell is computed once per CTA into
    // the staged tile; stored input: neighbours straight from L1
    return launch_zmarch<MsrOp<MODE, RC, DM>, RC>(g, name, op, pgeo(f, p), zb, ze);
}

// halo of the map output after the boundary maps on the halo stream (NCCL
// across processes, device copies within one), overlapped with the internal
// work of the compute stream and joined by an event before the boundary
// stencils


// mark: the boundary maps are enqueued (event eb on the compute stream);
// begin: the halo stream waits for eb and transfers.  Between the two the
// internal stencils are enqueued, so the host never holds them back behind
// the transfer's API calls.
static nb_status dist_halo_mark(nb_grid *g, HaloSync &hsync) {
    if (!nb_halo_on_stream(g)) return NB_OK;  // (peer transport: nothing to mark)
    if (!hsync.eb) {
        NB_CUDA(cudaEventCreateWithFlags(&hsync.eb, cudaEventDisableTiming));
        NB_CUDA(cudaEventCreateWithFlags(&hsync.eh, cudaEventDisableTiming));
    }
    NB_CUDA(cudaEventRecord(hsync.eb, g->cs));
    return NB_OK;
}
static nb_status dist_halo_begin(nb_grid *g, nb_field *u, HaloSync &hsync) {
    // peer transport: the boundary maps already stored the halo into the
    // neighbours; tell them
    if (!nb_halo_on_stream(g)) return nb_is_peer(g) ? nb_peer_signal(g, false, g->cs) : NB_OK;
    NB_CUDA(cudaStreamWaitEvent(g->hs, hsync.eb, 0));
    NB_TRY(nb_halo_exchange_planes(u, 0, 1, true, true, g->hs));
    NB_CUDA(cudaEventRecord(hsync.eh, g->hs));
    return NB_OK;
}
static nb_status dist_halo_wait(nb_grid *g, HaloSync &hsync) {
    if (!nb_halo_on_stream(g)) return nb_is_peer(g) ? nb_peer_wait(g, false, g->cs) : NB_OK;
    NB_CUDA(cudaStreamWaitEvent(g->cs, hsync.eh, 0));
    return NB_OK;
}

// per-partition arguments: MsrArgs holds partition pointers, so the step is
// run partition by partition through this adaptor
struct MsrFields {
    const nb_field *w, *v;
    nb_field *u, *out, *xs;
};

template <int MODE>
static nb_status msr_step_fields(nb_grid *g, nb_occ occ, MsrFields F, double m, double ap, int pending,
                                 const CgScal *sc, HaloSync &hs) {
    // maps
    auto args = [&](int p) {
        MsrArgs A;
        A.w = (const double *)F.w->base[p];
        A.v = (const double *)F.v->base[p];
        A.u = (double *)F.u->base[p];
        A.out = F.out ? (double *)F.out->base[p] : nullptr;
        A.xs = F.xs ? (double *)F.xs->base[p] : nullptr;
        A.m = m;
        A.ap = ap;
        A.pending = pending;
        A.sc = sc;
        return A;
    };
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbPart &q = g->parts[p];
        if (occ == NB_OCC_NONE || occ == NB_OCC_STANDARD) {
            NB_TRY(launch_map_u(g, MODE, p, args(p), F.u, 0, q.nz()));
        } else {
            const auto bp = bnd_pair(g, p);  // both boundary planes in one launch
            if (bp.first >= 0) NB_TRY(launch_map_u(g, MODE, p, args(p), F.u, bp.first, bp.first + 1, bp.second));
        }
    }
    NB_TRY(dist_halo_mark(g, hs));
    if (occ == NB_OCC_NONE) {
        NB_TRY(dist_halo_begin(g, F.u, hs));
        NB_TRY(dist_halo_wait(g, hs));
    }
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        auto in = view_ranges(g, p, occ == NB_OCC_NONE ? NB_VIEW_STANDARD : NB_VIEW_INTERNAL);
        for (auto rg : in) {
            if (occ == NB_OCC_NONE || occ == NB_OCC_STANDARD)
                NB_TRY((launch_msr<MODE, false, false>(g, p, args(p), F.u, rg.first, rg.second)));
            else
                NB_TRY((launch_msr<MODE, true, true>(g, p, args(p), F.u, rg.first, rg.second)));
        }
    }
    if (occ == NB_OCC_NONE) return NB_OK;
    NB_TRY(dist_halo_begin(g, F.u, hs));
    NB_TRY(dist_halo_wait(g, hs));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const auto bp = bnd_pair(g, p);  // both boundary planes in one launch where the kernel takes pairs
        if (bp.first < 0) continue;
        if (occ == NB_OCC_STANDARD)
            NB_TRY((launch_msr<MODE, false, false>(g, p, args(p), F.u, bp.first, bp.first + 1, bp.second)));
        else
            NB_TRY((launch_msr<MODE, true, false>(g, p, args(p), F.u, bp.first, bp.first + 1, bp.second)));
    }
    return NB_OK;
}

// ===========================================================================
// config C1: map -> stencil -> reduce loop (Fig. 4a)
// ===========================================================================
extern "C" nb_status nb_map_stencil_reduce(nb_field *x, nb_field *y, double a, int32_t iters, nb_occ occ,
                                           double *dots_out) {
    NB_RANGE("nb_map_stencil_reduce");
    if (!x || !y || !dots_out) NB_FAIL(NB_EINVAL, "nb_map_stencil_reduce: NULL argument");
    if (x->g != y->g) NB_FAIL(NB_EMISMATCH, "fields belong to different grids");
    if (x->dt != NB_F64 || y->dt != NB_F64 || x->card != 1 || y->card != 1)
        NB_FAIL(NB_EMISMATCH, "nb_map_stencil_reduce needs scalar fp64 fields");
    if (iters < 0 || iters > NB_DOT_SLOTS) NB_FAIL(NB_EINVAL, "iters must be in [0, %d]", NB_DOT_SLOTS);
    if (occ < NB_OCC_NONE || occ > NB_OCC_TWO_WAY) NB_FAIL(NB_EINVAL, "bad occ");
    nb_grid *g = x->g;
    if (g->sparse) NB_FAIL(NB_EUNSUPPORTED, "nb_map_stencil_reduce: dense grids only");
    if (x->outside != 0.0) NB_FAIL(NB_EUNSUPPORTED, "nb_map_stencil_reduce: outside value must be 0");
    cudaSetDevice(g->device);
    // ping-pong partners (the stencil reads neighbours of x and y while the
    // step writes new x and y)
    nb_field *x2 = nullptr, *y2 = nullptr;
    NB_TRY(nb_grid_scratch(g, NB_F64, 1, 0, &x2));
    nb_status st = nb_grid_scratch(g, NB_F64, 1, 1, &y2);
    HaloSync hs;
    nb_field *xin = x, *yin = y, *xo = x2, *yo = y2;
    // single process: every iteration writes its tile partials into its own
    // slice and ONE finalize produces all the dots (same trees, same bits as
    // a finalize per iteration); across processes, one finalize per iteration
    const bool defer = st == NB_OK && iters > 0 && !(g->comm && g->comm->world > 1) && !getenv("NB_C1_FIN_EACH");
    if (defer) {
        const int64_t need = (int64_t)iters * g->nz * g->T;
        if (g->c1_cap < need) {
            cudaFree(g->c1_tp);
            cudaFree(g->c1_psum);
            g->c1_tp = g->c1_psum = nullptr;
            g->c1_cap = 0;
            NB_CUDA(cudaMalloc(&g->c1_tp, sizeof(double) * need));
            NB_CUDA(cudaMalloc(&g->c1_psum, sizeof(double) * iters * g->nz));
            g->c1_cap = need;
        }
    }
    auto loop = [&]() -> nb_status {
        nb_status s = NB_OK;
        double *tp0 = g->tp;
        for (int k = 0; k < iters && s == NB_OK; ++k) {
            MsrFields F{xin, yin, xo, yo, nullptr};
            if (defer) g->tp = g->c1_tp + (int64_t)k * g->nz * g->T;  // this iteration's slice
            s = msr_step_fields<MSR_C1>(g, occ, F, a, 0.0, 0, nullptr, hs);
            g->tp = tp0;
            if (s == NB_OK && !defer) s = nb_reduce_finalize(g, 1, FIN_STORE, nullptr, k);
            std::swap(xin, xo);
            std::swap(yin, yo);
        }
        if (s == NB_OK && defer) s = nb_c1_finalize_all(g, iters);
        return s;
    };
    // the loop is launch-latency bound at small sizes (C1: 64^3): replay it
    // as one CUDA graph (rebuilt when fields, a, iterations or OCC change),
    // except under per-launch profiling, NCCL or event-ordered halo streams,
    // and across processes (the peer reductions alternate buffers by a host
    // counter that a replay would not advance)
    const bool graph = st == NB_OK && iters > 0 && !g->profiling && !nb_halo_on_stream(g) && !nb_is_peer(g) &&
                       !getenv("NB_NO_GRAPH");
    if (graph) {
        const int fl = g->first_local;
        const bool hit = g->c1_exec && g->c1_x == x->base[fl] && g->c1_y == y->base[fl] && g->c1_a == a &&
                         g->c1_iters == iters && g->c1_occ == (int)occ && g->c1_defer == (int)defer;
        if (!hit) {
            if (g->c1_exec) cudaGraphExecDestroy(g->c1_exec);
            g->c1_exec = nullptr;
            const int64_t l0 = g->launches;
            cudaGraph_t gr;
            NB_CUDA(cudaStreamBeginCapture(g->cs, cudaStreamCaptureModeThreadLocal));
            st = loop();
            cudaError_t e = cudaStreamEndCapture(g->cs, &gr);
            g->c1_launches = g->launches - l0;
            g->launches = l0;
            if (st == NB_OK && e != cudaSuccess) NB_FAIL(NB_ECUDA, "C1 graph capture: %s", cudaGetErrorString(e));
            if (st == NB_OK) {
                e = cudaGraphInstantiate(&g->c1_exec, gr, nb_graph_flags());
                cudaGraphDestroy(gr);
                if (e != cudaSuccess) NB_FAIL(NB_ECUDA, "C1 graph instantiate: %s", cudaGetErrorString(e));
                g->c1_x = x->base[fl];
                g->c1_y = y->base[fl];
                g->c1_a = a;
                g->c1_iters = iters;
                g->c1_occ = (int)occ;
                g->c1_defer = (int)defer;
            }
        } else {  // the replay ends where the captured loop ended
            for (int k = 0; k < iters; ++k) {
                std::swap(xin, xo);
                std::swap(yin, yo);
            }
        }
        if (st == NB_OK) {
            NB_CUDA(cudaGraphLaunch(g->c1_exec, g->cs));
            g->launches += g->c1_launches;
        }
    } else {
        st = loop();
    }
    if (st == NB_OK && xin != x) {  // odd iteration count: results live in the partners
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            size_t bytes = x->bytes[p];
            cudaMemcpyAsync(x->base[p], xin->base[p], bytes, cudaMemcpyDeviceToDevice, g->cs);
            cudaMemcpyAsync(y->base[p], yin->base[p], bytes, cudaMemcpyDeviceToDevice, g->cs);
        }
    }
    if (st == NB_OK && iters > 0) {
        cudaError_t e = cudaMemcpyAsync(dots_out, g->dots, sizeof(double) * iters, cudaMemcpyDeviceToHost, g->cs);
        if (e != cudaSuccess) {
            nb_set_error("cudaMemcpyAsync: %s", cudaGetErrorString(e));
            st = NB_ECUDA;
        }
    }
    cudaError_t e = cudaStreamSynchronize(g->cs);
    if (st == NB_OK && e != cudaSuccess) {
        nb_set_error("nb_map_stencil_reduce: %s", cudaGetErrorString(e));
        st = NB_ECUDA;
    }
    if (hs.eb) {
        cudaEventDestroy(hs.eb);
        cudaEventDestroy(hs.eh);
    }
    return st;
}

// ===========================================================================
// CG (Listing 3, UpdateP first L460) — two-phase schedule, 64 B/cell/iter:
//   phase A: p_new = r + beta p_old (recomputed at neighbours), x += alpha_prev
//            p_old (deferred), q = A p_new, <p_new, q>       40 B/cell
//   finalize: alpha = rr / <p,q>
//   phase B: q = A p_new (recomputed from stored p_new), r -= alpha q, <r,r>
//                                                            24 B/cell
//   finalize: beta = rr'/rr, ...
// ===========================================================================
nb_status nb_fem_cg_hooks(nb_cg *cg, int what);  // nb_fem.cu
nb_status nb_sparse_cg_hooks(nb_cg *cg, int what);

static nb_status cg_enqueue_iteration(nb_cg *cg) {
    nb_grid *g = cg->g;
    int64_t k = cg->k + 1;  // iteration number being enqueued
    nb_field *pn = cg->p[k & 1], *po = cg->p[(k + 1) & 1];
    if (cg->prm.op == NB_OP_FEM27) return nb_fem_cg_hooks(cg, (int)(k & 1));
    if (g->sparse) return nb_sparse_cg_hooks(cg, (int)(k & 1));
    // phase A (beta, alpha_prev and pending are read on the device from sc)
    MsrFields F{cg->r, po, pn, nullptr, cg->x};
    NB_TRY(msr_step_fields<MSR_CG>(g, cg->prm.occ, F, 0.0, 0.0, 0, cg->sc, cg->hs));
    NB_TRY(nb_reduce_finalize(g, 1, FIN_CG_PQ, cg->sc, 0));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        PGeo geo = pgeo(pn, p);
        if (ZR_STO == 1 && nb_tma_enabled()) {  // TMA-staged phase B
            NB_TRY(nb_cgB_tma(g, geo, (const double *)pn->base[p], (double *)cg->r->base[p], 0, geo.nzl, cg->sc));
            continue;
        }
        CgBOp op{(const double *)pn->base[p], (double *)cg->r->base[p], cg->sc, 0.0};
        NB_TRY(launch_zmarch(g, "k_cg_B", op, geo, 0, geo.nzl));
    }
    NB_TRY(nb_reduce_finalize(g, 1, FIN_CG_RR, cg->sc, 0));
    cg->k = k;
    return NB_OK;
}

static nb_status cg_check(const nb_field *x, const nb_field *b, const nb_cg_params *prm) {
    if (!x || !b || !prm) NB_FAIL(NB_EINVAL, "nb_cg: NULL argument");
    if (x->g != b->g) NB_FAIL(NB_EMISMATCH, "x and b belong to different grids");
    if (x->dt != NB_F64 || b->dt != NB_F64) NB_FAIL(NB_EMISMATCH, "CG runs in fp64");
    int card = prm->op == NB_OP_FEM27 ? 3 : 1;
    if (x->card != card || b->card != card) NB_FAIL(NB_EMISMATCH, "CG operator needs cardinality %d", card);
    if (x->layout != b->layout) NB_FAIL(NB_EMISMATCH, "x and b have different layouts");
    if (prm->op == NB_OP_FEM27) NB_LAYOUTS(x, (1 << NB_SOA) | (1 << NB_SOA_PLANE), "FEM CG");
    if (prm->op != NB_OP_LAPLACE7 && prm->op != NB_OP_FEM27) NB_FAIL(NB_EINVAL, "bad operator");
    if (prm->occ < NB_OCC_NONE || prm->occ > NB_OCC_TWO_WAY) NB_FAIL(NB_EINVAL, "bad occ");
    if (x->outside != 0.0) NB_FAIL(NB_EUNSUPPORTED, "CG: x must have outside value 0 (homogeneous Dirichlet)");
    return NB_OK;
}

nb_status nb_fem_cg_init(nb_cg *cg);           // nb_fem.cu
nb_status nb_sparse_cg_init(nb_cg *cg);        // nb_sparse.cu
nb_status nb_sparse_cg_flush(nb_cg *cg);

extern "C" nb_status nb_cg_create(nb_field *x, const nb_field *b, const nb_cg_params *prm, nb_cg **out) {
    NB_RANGE("nb_cg_create");
    if (!out) NB_FAIL(NB_EINVAL, "nb_cg_create: out is NULL");
    *out = nullptr;
    NB_TRY(cg_check(x, b, prm));
    nb_grid *g = x->g;
    cudaSetDevice(g->device);
    nb_cg *cg = new nb_cg();
    cg->g = g;
    cg->x = x;
    cg->b = b;
    cg->prm = *prm;
    int card = x->card;
    nb_status s = nb_field_create(g, NB_F64, card, x->layout, 0.0, &cg->r);
    if (s == NB_OK) s = nb_field_create(g, NB_F64, card, x->layout, 0.0, &cg->p[0]);
    if (s == NB_OK) s = nb_field_create(g, NB_F64, card, x->layout, 0.0, &cg->p[1]);
    if (s == NB_OK && (prm->op == NB_OP_FEM27 || g->sparse)) s = nb_field_create(g, NB_F64, card, x->layout, 0.0, &cg->q);
    if (s == NB_OK && cudaMalloc(&cg->sc, sizeof(CgScal)) != cudaSuccess) {
        nb_set_error("cudaMalloc scalars failed");
        s = NB_ENOMEM;
    }
    if (s == NB_OK) {
        CgScal h{};
        h.rtol2 = prm->rtol * prm->rtol;
        cudaMemcpyAsync(cg->sc, &h, sizeof(CgScal), cudaMemcpyHostToDevice, g->cs);
        // r = b - A x and rr0 (x's halo first)
        s = nb_halo_update(x);
        if (s == NB_OK) {
            if (prm->op == NB_OP_FEM27) {
                s = nb_fem_cg_init(cg);
            } else if (g->sparse) {
                s = nb_sparse_cg_init(cg);
            } else {
                for (int p = g->first_local; p < g->first_local + g->nlocal && s == NB_OK; ++p) {
                    PGeo geo = pgeo(x, p);
                    CgInitOp op{(const double *)x->base[p], (const double *)b->base[p], (double *)cg->r->base[p],
                                x->outside};
                    s = launch_zmarch(g, "k_cg_init", op, geo, 0, geo.nzl);
                }
                if (s == NB_OK) s = nb_reduce_finalize(g, 1, FIN_CG_INIT, cg->sc, 0);
            }
        }
    }
    g->nsolvers++;
    if (s != NB_OK) {
        nb_cg_destroy(cg);
        return s;
    }
    *out = cg;
    return NB_OK;
}

static bool cg_eager(const nb_grid *g) {
    return g->profiling || nb_is_nccl(g) || getenv("NB_NO_GRAPH") != nullptr;
}

constexpr int CG_GRAPH_CHUNK = 16;

// the CUDA graph of n iterations starting at parity `par` (captured once)
static nb_status cg_graph(nb_cg *cg, int n, int par, std::pair<cudaGraphExec_t, int64_t> **out) {
    nb_grid *g = cg->g;
    auto key = std::make_pair(n, par);
    auto it = cg->graphs.find(key);
    if (it == cg->graphs.end()) {
        cudaGraph_t graph;
        int64_t l0 = g->launches, k0 = cg->k;
        cg->k = par;  // parity of the first captured iteration is (par + 1) & 1
        NB_CUDA(cudaStreamBeginCapture(g->cs, cudaStreamCaptureModeThreadLocal));
        nb_status s = NB_OK;
        for (int i = 0; i < n && s == NB_OK; ++i) s = cg_enqueue_iteration(cg);
        cudaError_t e = cudaStreamEndCapture(g->cs, &graph);
        int64_t nl = g->launches - l0;
        g->launches = l0;
        cg->k = k0;
        if (s != NB_OK) return s;
        if (e != cudaSuccess) NB_FAIL(NB_ECUDA, "graph capture failed: %s", cudaGetErrorString(e));
        cudaGraphExec_t exec;
        e = cudaGraphInstantiate(&exec, graph, nb_graph_flags());
        cudaGraphDestroy(graph);
        if (e != cudaSuccess) NB_FAIL(NB_ECUDA, "graph instantiate failed: %s", cudaGetErrorString(e));
        it = cg->graphs.emplace(key, std::make_pair(exec, nl)).first;
    }
    *out = &it->second;
    return NB_OK;
}

// walk the chunks nb_cg_iterate(iters) will use; launch them or only build them
static nb_status cg_run_chunks(nb_cg *cg, int32_t iters, bool launch) {
    nb_grid *g = cg->g;
    int64_t k = cg->k;
    int done = 0;
    while (done < iters) {
        int n = std::min(CG_GRAPH_CHUNK, iters - done);
        std::pair<cudaGraphExec_t, int64_t> *gr = nullptr;
        NB_TRY(cg_graph(cg, n, (int)(k & 1), &gr));
        if (launch) {
            NB_CUDA(cudaGraphLaunch(gr->first, g->cs));
            g->launches += gr->second;
        }
        k += n;
        done += n;
    }
    if (launch) cg->k = k;
    return NB_OK;
}

extern "C" nb_status nb_cg_iterate(nb_cg *cg, int32_t iters) {
    NB_RANGE("nb_cg_iterate");
    if (!cg) NB_FAIL(NB_EINVAL, "nb_cg_iterate: NULL solver");
    if (cg->finished) NB_FAIL(NB_ESTATE, "nb_cg_iterate after nb_cg_finish");
    if (iters < 0) NB_FAIL(NB_EINVAL, "iters < 0");
    nb_grid *g = cg->g;
    cudaSetDevice(g->device);
    if (cg_eager(g)) {  // profiling (per-launch events) or multi-process (NCCL inside)
        for (int i = 0; i < iters; ++i) NB_TRY(cg_enqueue_iteration(cg));
        return NB_OK;
    }
    return cg_run_chunks(cg, iters, true);
}

extern "C" nb_status nb_cg_prepare(nb_cg *cg, int32_t iters) {
    if (!cg) NB_FAIL(NB_EINVAL, "nb_cg_prepare: NULL solver");
    if (iters < 0) NB_FAIL(NB_EINVAL, "iters < 0");
    cudaSetDevice(cg->g->device);
    if (cg_eager(cg->g)) return NB_OK;
    return cg_run_chunks(cg, iters, false);
}

extern "C" nb_status nb_cg_finish(nb_cg *cg, nb_cg_result *res) {
    if (!cg) NB_FAIL(NB_EINVAL, "nb_cg_finish: NULL solver");
    nb_grid *g = cg->g;
    cudaSetDevice(g->device);
    if (!cg->finished) {
        if (g->sparse) {  // one p buffer (Poisson and FEM)
            NB_TRY(nb_sparse_cg_flush(cg));
        } else {
            for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
                int64_t n = (int64_t)cg->x->bytes[p] / 8;
                LaunchScope ls(g, g->cs, "k_cg_flush");
                // p ping-pongs by iteration parity (dense Poisson and FEM)
                const double *p1 = (const double *)cg->p[1]->base[p];
                k_cg_flush<<<148 * 4, 256, 0, g->cs>>>((double *)cg->x->base[p], (const double *)cg->p[0]->base[p], p1,
                                                      n, cg->sc);
                NB_TRY(nb_launch_check("k_cg_flush"));
            }
        }
        k_cg_flush_done<<<1, 32, 0, g->cs>>>(cg->sc);
        NB_TRY(nb_launch_check("k_cg_flush_done"));
        cg->finished = true;
    }
    CgScal h;
    NB_CUDA(cudaMemcpyAsync(&h, cg->sc, sizeof(CgScal), cudaMemcpyDeviceToHost, g->cs));
    NB_CUDA(cudaStreamSynchronize(g->cs));
    if (res) {
        res->iters = h.iters;
        res->converged = h.status;
        res->rr0 = h.rr0;
        res->rr = h.rr;
    }
    return NB_OK;
}

nb_status nb_cg_status(nb_cg *cg, int *status, int *iters) {
    CgScal h;
    NB_CUDA(cudaMemcpyAsync(&h, cg->sc, sizeof(CgScal), cudaMemcpyDeviceToHost, cg->g->cs));
    NB_CUDA(cudaStreamSynchronize(cg->g->cs));
    *status = h.status;
    *iters = h.iters;
    return NB_OK;
}

extern "C" nb_status nb_cg_destroy(nb_cg *cg) {
    if (!cg) return NB_OK;
    cudaSetDevice(cg->g->device);
    cudaStreamSynchronize(cg->g->cs);
    for (auto &kv : cg->graphs) cudaGraphExecDestroy(kv.second.first);
    if (cg->hs.eb) {
        cudaEventDestroy(cg->hs.eb);
        cudaEventDestroy(cg->hs.eh);
    }
    nb_field_destroy(cg->r);
    nb_field_destroy(cg->p[0]);
    nb_field_destroy(cg->p[1]);
    nb_field_destroy(cg->q);
    if (cg->sc) cudaFree(cg->sc);
    cg->g->nsolvers--;
    delete cg;
    return NB_OK;
}

extern "C" nb_status nb_cg_solve(nb_field *x, const nb_field *b, const nb_cg_params *prm, nb_cg_result *res) {
    nb_cg *cg = nullptr;
    NB_TRY(nb_cg_create(x, b, prm, &cg));
    int every = prm->check_every > 0 ? prm->check_every : 16;
    int done = 0;
    nb_status s = NB_OK;
    while (done < prm->max_iter && s == NB_OK) {
        int n = std::min(every, prm->max_iter - done);
        s = nb_cg_iterate(cg, n);
        done += n;
        if (s == NB_OK && prm->rtol > 0.0 && done < prm->max_iter) {
            int st = 0, it = 0;
            s = nb_cg_status(cg, &st, &it);
            if (st != 0) break;
        }
    }
    if (s == NB_OK) s = nb_cg_finish(cg, res);
    nb_cg_destroy(cg);
    return s;
}
