// nb_tma.cu — TMA-staged CG phase A (the headline hot kernel).
//
// Same arithmetic and canonical dot order as k_msr_fast<MSR_CG, DOMAP> (and
// k_zmarch<MsrOp<MSR_CG, true, DOMAP>>): p_new = fma(beta, p_old, r) for
// every cell of the tile and its ring, x += alpha_prev p_old (deferred),
// q = fma(6, p_new_c, -s), per-plane tile partial of p_new * q.
//
// Data movement is Blackwell-native: one elected thread issues, per plane, a
// 3-D TMA box load (cp.async.bulk.tensor) of the 36 x 10 (tile + ring) box of
// r and of p_old — or of the stored p_new on halo planes — plus the 32 x 8
// box of x, into a 4-stage shared-memory ring completed through mbarriers
// (transaction bytes).  Out-of-domain x/y cells of the box are zero-filled by
// the TMA unit, which is exactly the outside value 0.  Planes are fetched
// two to three steps ahead, so the per-plane barrier rarely waits on DRAM.
#include <cuda.h>

#include <cstring>
#include <map>
#include <mutex>
#include <tuple>

#include "nb_device.cuh"
#include "nb_internal.cuh"
#include "nb_tma.cuh"

#ifndef NB_ZC
#define NB_ZC 32
#endif
constexpr int TZC = NB_ZC;  // planes per CTA (matches the z-march chunking)
// the box starts at x0 - 2: TMA needs the innermost start coordinate 16-byte
// aligned (even for fp64), so the x ring is 2 cells wide on the left
constexpr int BX = DOT_TX + 4, BY = DOT_TY + 2;
constexpr int TPAD = 2944;  // tile bytes rounded up to 128
constexpr int NSTAGE = 4;

struct __align__(128) CgAStage {
    double a[BY][BX];  // r (in-slab planes) or stored p_new (halo planes)
    double pad0[(TPAD - BY * BX * 8) / 8];
    double b[BY][BX];  // p_old
    double pad1[(TPAD - BY * BX * 8) / 8];
    double xs[DOT_TY][DOT_TX];  // x of the own cells
};
static_assert(sizeof(double) * BY * BX < TPAD && TPAD % 128 == 0, "stage tile padding");

// C1 (C1 = true): the same map -> stencil -> reduce chain of Fig. 4a with
// r -> x_in, p_old -> y_in, p_new -> x_out (u = fma(a, y_in, x_in)),
// out = L(u) = fma(-6, u, s) stored to y_out, dot u * out, no deferred x.
template <bool DOMAP, bool C1 = false>
__global__ void __launch_bounds__(DOT_TX *DOT_TY)
    k_cgA_tma(const __grid_constant__ CUtensorMap m_r, const __grid_constant__ CUtensorMap m_po,
              const __grid_constant__ CUtensorMap m_pn, const __grid_constant__ CUtensorMap m_x, double *pn, double *xs,
              PGeo g, int zb, int ze, const CgScal *sc, double *tp, int T, int tiles_y, int zc, double c1_a = 0.0,
              double *c1_out = nullptr) {
    __shared__ CgAStage st[NSTAGE];
    __shared__ __align__(8) uint64_t bar[NSTAGE];
    __shared__ double sw[TZC][DOT_TY];
    if (!C1 && sc->status != 0) return;
    const double beta = C1 ? c1_a : sc->beta, ap = C1 ? 0.0 : sc->alpha_prev;
    const bool dox = !C1 && DOMAP && sc->pending;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const int x0 = blockIdx.x * DOT_TX, y0 = blockIdx.y * DOT_TY;
    const int xi = x0 + lane, yi = y0 + w;
    const int zs = zb + blockIdx.z * zc, zend = min(ze, zs + zc);  // zc <= TZC planes per CTA
    const int nzl = g.nzl;
    const bool valid = xi < g.nx && yi < g.ny;
    auto halo = [&](int zl) { return zl < 0 || zl >= nzl; };
    auto stage_of = [&](int zl) { return (zl - zs + 1) & (NSTAGE - 1); };
    auto parity_of = [&](int zl) { return (uint32_t)(((zl - zs + 1) / NSTAGE) & 1); };
    // producer: one thread fetches plane zl into its stage
    auto issue = [&](int zl) {
        CgAStage &s = st[stage_of(zl)];
        uint64_t *b = &bar[stage_of(zl)];
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        if (halo(zl)) {
            mbar_expect_tx(b, BY * BX * 8);
            tma_load_3d(&s.a[0][0], &m_pn, b, x0 - 2, y0 - 1, zl + 1);
        } else {
            const bool wx = dox && zl >= zs && zl < zend;
            mbar_expect_tx(b, 2 * BY * BX * 8 + (wx ? DOT_TY * DOT_TX * 8 : 0));
            tma_load_3d(&s.a[0][0], &m_r, b, x0 - 2, y0 - 1, zl + 1);
            tma_load_3d(&s.b[0][0], &m_po, b, x0 - 2, y0 - 1, zl + 1);
            if (wx) tma_load_3d(&s.xs[0][0], &m_x, b, x0, y0, zl + 1);
        }
    };
    if (tid == 0) {
        for (int k = 0; k < NSTAGE; ++k) mbar_init(&bar[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (tid == 0)
        for (int zl = zs - 1; zl <= min(zs + 2, zend); ++zl) issue(zl);
    // p_new at tile cell (yy, xx) of plane zl's stage
    auto U = [&](int zl, int yy, int xx) -> double {
        const CgAStage &s = st[stage_of(zl)];
        return halo(zl) ? s.a[yy][xx] : fma(beta, s.b[yy][xx], s.a[yy][xx]);
    };
    mbar_wait(&bar[stage_of(zs - 1)], parity_of(zs - 1));
    mbar_wait(&bar[stage_of(zs)], parity_of(zs));
    double below = U(zs - 1, w + 1, lane + 2);
    double center = U(zs, w + 1, lane + 2);
    const int64_t o = (int64_t)yi * g.pitch + xi + g.ps;  // (xi, yi, zl = 0)
    for (int z = zs; z < zend; ++z) {
        // one thread waits on the stage's mbarrier, the CTA barrier releases
        // the others (no per-thread try_wait polling); the stage of plane
        // z-1 is free once every thread passed this barrier
        if (tid == 0) mbar_wait(&bar[stage_of(z + 1)], parity_of(z + 1));
        __syncthreads();
        if (tid == 0 && z + 3 <= zend) issue(z + 3);  // -> stage of plane z-1 (read before this barrier)
        const double above = U(z + 1, w + 1, lane + 2);
        double prod = 0.0;
        if (valid) {
            double s = __dadd_rn(U(z, w + 1, lane + 1), U(z, w + 1, lane + 3));
            s = __dadd_rn(s, U(z, w, lane + 2));
            s = __dadd_rn(s, U(z, w + 2, lane + 2));
            s = __dadd_rn(s, below);
            s = __dadd_rn(s, above);
            const double q = C1 ? fma(-6.0, center, s) : fma(6.0, center, -s);
            const int64_t e = o + (int64_t)z * g.ps;
            if (C1) __stcs(c1_out + e, q);
            if (DOMAP) {
                pn[e] = center;
                if (dox) {
                    const CgAStage &sz = st[stage_of(z)];
                    xs[e] = fma(ap, sz.b[w + 1][lane + 2], sz.xs[w][lane]);
                }
            }
            prod = __dmul_rn(center, q);
        }
        prod = warp_sum_canon(prod);
        if (lane == 0) sw[z - zs][w] = prod;
        below = center;
        center = above;
    }
    __syncthreads();  // sw complete
    // per-plane tile partials: the 8 row values in increasing y
    if (tid < zend - zs) {
        double s = sw[tid][0];
#pragma unroll
        for (int k = 1; k < DOT_TY; ++k) s = __dadd_rn(s, sw[tid][k]);
        tp[((int64_t)g.z0 + zs + tid) * T + blockIdx.y * gridDim.x + blockIdx.x] = s;
    }
}

// ---------------------------------------------------------------------------
// CG phase B, TMA-staged: q = A p_new from the stored p_new (36 x 10 box per
// plane, halo planes included), r -= alpha q (32 x 8 box of r per plane),
// per-plane tile partial of r*r in the ZR = 1 canonical order (butterfly per
// row, rows in increasing y).
// ---------------------------------------------------------------------------
struct __align__(128) CgBStage {
    double p[BY][BX];
    double pad0[(TPAD - BY * BX * 8) / 8];
    double r[DOT_TY][DOT_TX];
};

__global__ void __launch_bounds__(DOT_TX *DOT_TY)
    k_cgB_tma(const __grid_constant__ CUtensorMap m_p, const __grid_constant__ CUtensorMap m_r, double *r, PGeo g,
              int zb, int ze, const CgScal *sc, double *tp, int T, int zc) {
    __shared__ CgBStage st[NSTAGE];
    __shared__ __align__(8) uint64_t bar[NSTAGE];
    __shared__ double sw[TZC][DOT_TY];
    if (sc->status != 0) return;
    const double alpha = sc->alpha;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const int x0 = blockIdx.x * DOT_TX, y0 = blockIdx.y * DOT_TY;
    const int xi = x0 + lane, yi = y0 + w;
    const int zs = zb + blockIdx.z * zc, zend = min(ze, zs + zc);
    const bool valid = xi < g.nx && yi < g.ny;
    auto stage_of = [&](int zl) { return (zl - zs + 1) & (NSTAGE - 1); };
    auto parity_of = [&](int zl) { return (uint32_t)(((zl - zs + 1) / NSTAGE) & 1); };
    auto issue = [&](int zl) {
        CgBStage &s = st[stage_of(zl)];
        uint64_t *b = &bar[stage_of(zl)];
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        const bool wr = zl >= zs && zl < zend;
        mbar_expect_tx(b, BY * BX * 8 + (wr ? DOT_TY * DOT_TX * 8 : 0));
        tma_load_3d(&s.p[0][0], &m_p, b, x0 - 2, y0 - 1, zl + 1);
        if (wr) tma_load_3d(&s.r[0][0], &m_r, b, x0, y0, zl + 1);
    };
    if (tid == 0) {
        for (int k = 0; k < NSTAGE; ++k) mbar_init(&bar[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (tid == 0)
        for (int zl = zs - 1; zl <= min(zs + 2, zend); ++zl) issue(zl);
    mbar_wait(&bar[stage_of(zs - 1)], parity_of(zs - 1));
    mbar_wait(&bar[stage_of(zs)], parity_of(zs));
    double below = st[stage_of(zs - 1)].p[w + 1][lane + 2];
    double center = st[stage_of(zs)].p[w + 1][lane + 2];
    const int64_t o = (int64_t)yi * g.pitch + xi + g.ps;
    for (int z = zs; z < zend; ++z) {
        if (tid == 0) mbar_wait(&bar[stage_of(z + 1)], parity_of(z + 1));
        __syncthreads();
        if (tid == 0 && z + 3 <= zend) issue(z + 3);  // -> stage of plane z-1 (read before this barrier)
        const CgBStage &sz = st[stage_of(z)];
        const double above = st[stage_of(z + 1)].p[w + 1][lane + 2];
        double prod = 0.0;
        if (valid) {
            double s = __dadd_rn(sz.p[w + 1][lane + 1], sz.p[w + 1][lane + 3]);
            s = __dadd_rn(s, sz.p[w][lane + 2]);
            s = __dadd_rn(s, sz.p[w + 2][lane + 2]);
            s = __dadd_rn(s, below);
            s = __dadd_rn(s, above);
            const double q = fma(6.0, center, -s);
            const double rn = fma(-alpha, q, sz.r[w][lane]);
            __stcs(r + o + (int64_t)z * g.ps, rn);
            prod = __dmul_rn(rn, rn);
        }
        prod = warp_sum_canon(prod);
        if (lane == 0) sw[z - zs][w] = prod;
        below = center;
        center = above;
    }
    __syncthreads();
    if (tid < zend - zs) {
        double s = sw[tid][0];
#pragma unroll
        for (int k = 1; k < DOT_TY; ++k) s = __dadd_rn(s, sw[tid][k]);
        tp[((int64_t)g.z0 + zs + tid) * T + blockIdx.y * gridDim.x + blockIdx.x] = s;
    }
}

// ---------------------------------------------------------------------------
// host side: tensor maps (cached per buffer and geometry)
// ---------------------------------------------------------------------------
// planes per CTA: TZC, halved while the launch would have fewer than two
// CTAs per SM (small grids, e.g. C1's 64^3: 16 tiles x 2 chunks = 32 CTAs);
// the dot partials are per plane and tile, so results do not depend on it
static int tma_zc(const nb_grid *g, int nplanes) {
    const int64_t tiles = (int64_t)g->tiles_x * g->tiles_y;
    int zc = TZC;
    while (zc > 2 && tiles * ((nplanes + zc - 1) / zc) < 2 * 148) zc /= 2;
    return zc;
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                  const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
    static EncodeTiledFn fn = nullptr;
    static bool tried = false;
    if (!tried) {
        tried = true;
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (EncodeTiledFn)p;
        else
            cudaGetLastError();
    }
    return fn;
}

static std::mutex g_tmap_mu;
static std::map<std::tuple<const void *, int, int, int, int64_t, int>, CUtensorMap> g_tmaps;

// box: 0 = (tile + ring) 36 x 10 x 1 (x from x0-2), 1 = own tile 32 x 8 x 1
nb_status tmap_for(const void *base, const PGeo &g, int box, CUtensorMap *out) {
    std::lock_guard<std::mutex> lk(g_tmap_mu);
    auto key = std::make_tuple(base, g.nx, g.ny, g.nzl, g.pitch, box);
    auto it = g_tmaps.find(key);
    if (it != g_tmaps.end()) {
        *out = it->second;
        return NB_OK;
    }
    EncodeTiledFn fn = encode_fn();
    if (!fn) NB_FAIL(NB_EUNSUPPORTED, "cuTensorMapEncodeTiled unavailable");
    CUtensorMap m;
    cuuint64_t dims[3] = {(cuuint64_t)g.nx, (cuuint64_t)g.ny, (cuuint64_t)(g.nzl + 2)};
    cuuint64_t strides[2] = {(cuuint64_t)g.pitch * 8, (cuuint64_t)g.ps * 8};
    cuuint32_t boxd[3] = {box == 0 ? (cuuint32_t)BX : (cuuint32_t)DOT_TX, box == 0 ? (cuuint32_t)BY : (cuuint32_t)DOT_TY,
                          1};
    cuuint32_t es[3] = {1, 1, 1};
    CUresult r = fn(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, const_cast<void *>(base), dims, strides, boxd, es,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) NB_FAIL(NB_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
    g_tmaps[key] = m;
    *out = m;
    return NB_OK;
}

// drop cached maps of a freed buffer
void nb_tma_forget(const void *base) {
    std::lock_guard<std::mutex> lk(g_tmap_mu);
    for (auto it = g_tmaps.begin(); it != g_tmaps.end();)
        it = std::get<0>(it->first) == base ? g_tmaps.erase(it) : std::next(it);
}

bool nb_tma_enabled() {
    static int en = -1;
    if (en < 0) en = getenv("NB_NO_TMA") ? 0 : 1;
    return en && encode_fn() != nullptr;
}

// CG phase A on planes [zb, ze) of a partition (r, p_old, p_new, x buffers)
nb_status nb_cgA_tma(nb_grid *g, const PGeo &geo, const double *r, const double *po, double *pn, double *x, bool domap,
                     int zb, int ze, const CgScal *sc) {
    if (ze <= zb) return NB_OK;
    CUtensorMap mr, mpo, mpn, mx;
    NB_TRY(tmap_for(r, geo, 0, &mr));
    NB_TRY(tmap_for(po, geo, 0, &mpo));
    NB_TRY(tmap_for(pn, geo, 0, &mpn));
    NB_TRY(tmap_for(x, geo, 1, &mx));
    const int zc = tma_zc(g, ze - zb);
    dim3 blk(DOT_TX * DOT_TY), grd(g->tiles_x, g->tiles_y, (ze - zb + zc - 1) / zc);
    LaunchScope ls(g, g->cs, "k_msr_cgA");
    if (domap)
        k_cgA_tma<true><<<grd, blk, 0, g->cs>>>(mr, mpo, mpn, mx, pn, x, geo, zb, ze, sc, g->tp, g->T, g->tiles_y, zc);
    else
        k_cgA_tma<false><<<grd, blk, 0, g->cs>>>(mr, mpo, mpn, mx, pn, x, geo, zb, ze, sc, g->tp, g->T, g->tiles_y, zc);
    return nb_launch_check("k_cgA_tma");
}

// C1 map-stencil-reduce on planes [zb, ze): x_out = x_in + a y_in (stored
// when domap), y_out = L(x_out), per-plane tile partials of x_out * y_out
nb_status nb_c1_tma(nb_grid *g, const PGeo &geo, const double *xin, const double *yin, double *xout, double *yout,
                    double a, bool domap, int zb, int ze) {
    if (ze <= zb) return NB_OK;
    CUtensorMap mx, my, mu;
    NB_TRY(tmap_for(xin, geo, 0, &mx));
    NB_TRY(tmap_for(yin, geo, 0, &my));
    NB_TRY(tmap_for(xout, geo, 0, &mu));
    const int zc = tma_zc(g, ze - zb);
    dim3 blk(DOT_TX * DOT_TY), grd(g->tiles_x, g->tiles_y, (ze - zb + zc - 1) / zc);
    LaunchScope ls(g, g->cs, "k_msr_c1");
    if (domap)
        k_cgA_tma<true, true><<<grd, blk, 0, g->cs>>>(mx, my, mu, mx, xout, nullptr, geo, zb, ze, nullptr, g->tp, g->T,
                                                      g->tiles_y, zc, a, yout);
    else
        k_cgA_tma<false, true><<<grd, blk, 0, g->cs>>>(mx, my, mu, mx, xout, nullptr, geo, zb, ze, nullptr, g->tp,
                                                       g->T, g->tiles_y, zc, a, yout);
    return nb_launch_check("k_c1_tma");
}

// CG phase B on planes [zb, ze) of a partition (stored p_new, r)
nb_status nb_cgB_tma(nb_grid *g, const PGeo &geo, const double *p, double *r, int zb, int ze, const CgScal *sc) {
    if (ze <= zb) return NB_OK;
    CUtensorMap mp, mr;
    NB_TRY(tmap_for(p, geo, 0, &mp));
    NB_TRY(tmap_for(r, geo, 1, &mr));
    const int zc = tma_zc(g, ze - zb);
    dim3 blk(DOT_TX * DOT_TY), grd(g->tiles_x, g->tiles_y, (ze - zb + zc - 1) / zc);
    LaunchScope ls(g, g->cs, "k_cg_B");
    k_cgB_tma<<<grd, blk, 0, g->cs>>>(mp, mr, r, geo, zb, ze, sc, g->tp, g->T, zc);
    return nb_launch_check("k_cgB_tma");
}
