// nb_tma.cu — TMA-staged CG phase A (the headline hot kernel).
//
// Same arithmetic and canonical dot order as k_msr_fast<MSR_CG, DOMAP> (and
// k_zmarch<MsrOp<MSR_CG, true, DOMAP>>): p_new = fma(beta, p_old, r) for
// every cell of the tile and its ring, x += alpha_prev p_old (deferred),
// q = fma(6, p_new_c, -s), per-plane tile partial of p_new * q.
//
// Data movement is Blackwell-native: a CTA covers two 32 x 8 dot tiles side
// by side (64 x 8 cells, 16 warps); one thread issues, per plane, a 3-D TMA
// box load (cp.async.bulk.tensor) of the 68 x 10 (tile + ring) box of r and
// of p_old — or of the stored p_new on halo planes — plus the 64 x 8 box of
// x, into a 4-stage shared-memory ring completed through mbarriers
// (transaction bytes).  Out-of-domain x/y cells of the box are zero-filled by
// the TMA unit, which is exactly the outside value 0.  Planes are fetched
// two to three steps ahead; the same thread polls the mbarrier and the CTA
// barrier releases the others.  The 64-wide CTA re-reads 1.33x its cells
// from L2 (1.41x for 32 x 8) and draws less power: under the board's power
// cap the CG step is 4 % faster than with 32 x 8 CTAs (same bits).
#include <cuda.h>

#include <cstring>
#include <map>
#include <mutex>
#include <tuple>
#include <queue>
#include <vector>

#include "nb_device.cuh"
#include "nb_internal.cuh"
#include "nb_tma.cuh"

#ifndef NB_ZC
#define NB_ZC 32
#endif
constexpr int TZC = NB_ZC;  // planes per CTA (matches the z-march chunking)
// A CTA covers NTX dot tiles side by side (32 NTX x 8 cells; warp w = row
// w % 8 of tile w / 8).  The box starts at x0 - 2: TMA needs the innermost
// start coordinate 16-byte aligned (even for fp64), so the x ring is 2 cells
// wide on the left: a (32 NTX + 4) x 10 box per plane.
#ifndef NB_CG_NTX
#define NB_CG_NTX 2  // dot tiles per CTA along x of the CG phases (2: 64 x 8 cells, 68 x 10 boxes)
#endif
#ifndef NB_CG_NTY
#define NB_CG_NTY 1  // dot tiles per CTA along y
#endif
#ifndef NB_CG_NST
#define NB_CG_NST 4  // ring stages
#endif
template <int NTX, int NTY = 1, int NST_ = 4>
struct TmaGeo {
    static constexpr int NST = NST_;                             // ring stages
    static constexpr int TW = DOT_TX * NTX;                      // CTA width (cells)
    static constexpr int TH = DOT_TY * NTY;                      // CTA height (rows)
    static constexpr int BXW = TW + 4;                           // box width
    static constexpr int BYH = TH + 2;                           // box height
    static constexpr int BOX = BYH * BXW;                        // box cells
    static constexpr int BPAD = (BOX * 8 + 127) / 128 * 128 / 8;  // box stride (doubles, 128-B aligned)
    static constexpr int OWN = TH * TW;                          // own-cell box
    static constexpr int NT = TW * TH;                           // threads
    static constexpr int SA = 2 * BPAD + OWN;                    // phase A stage (doubles)
    static constexpr int SB = BPAD + OWN;                        // phase B stage
    // CTAs per SM the registers must allow: as many as the shared memory
    // does (ring + ~5 KB static + 1 KB reserved per CTA of 228 KB per SM)
    static constexpr int fit(int ring) {
        const int by_smem = 233472 / (ring * 8 + 6 * 1024), by_threads = 2048 / NT;
        return by_smem < by_threads ? by_smem : by_threads;
    }
    static constexpr int MINB_A = fit(NST * SA), MINB_B = fit(NST * SB);
};
using CgGeo = TmaGeo<NB_CG_NTX, NB_CG_NTY, NB_CG_NST>;

// C1 (C1 = true): the same map -> stencil -> reduce chain of Fig. 4a with
// r -> x_in, p_old -> y_in, p_new -> x_out (u = fma(a, y_in, x_in)),
// out = L(u) = fma(-6, u, s) stored to y_out, dot u * out, no deferred x.
// Stage layout (dynamic shared memory): a = r (in-slab planes) or the stored
// p_new (halo planes), b = p_old, then x of the own cells.
template <bool DOMAP, bool C1, class G>
__global__ void __launch_bounds__(G::NT, G::MINB_A)
    k_cgA_tma(const __grid_constant__ CUtensorMap m_r, const __grid_constant__ CUtensorMap m_po,
              const __grid_constant__ CUtensorMap m_pn, const __grid_constant__ CUtensorMap m_x, double *pn, double *xs,
              PGeo g, int zb, int ze, const CgScal *sc, double *tp, int T, int tiles_x, int zc, double c1_a,
              double *c1_out, int zhi) {
    constexpr int NTX = G::TW / DOT_TX, NTY = G::TH / DOT_TY, NSTAGE = G::NST;
    extern __shared__ __align__(128) double tsm[];
    __shared__ __align__(8) uint64_t bar[NSTAGE];
    __shared__ double sw[TZC][NTY * NTX][DOT_TY];
    pdl_wait();  // the previous kernel's scalars and fields (programmatic launch)
    if (!C1 && sc->status != 0) return;
    const double beta = C1 ? c1_a : sc->beta, ap = C1 ? 0.0 : sc->alpha_prev;
    const bool dox = !C1 && DOMAP && sc->pending;
    // warp -> (dot tile t = (ty, tx) of the CTA, row wr of that tile); w = CTA row
    const int tid = threadIdx.x, lane = tid & 31, wr = (tid >> 5) % DOT_TY, t = (tid >> 5) / DOT_TY;
    const int tx = t % NTX, ty = t / NTX, w = ty * DOT_TY + wr;
    const int x0 = blockIdx.x * G::TW, y0 = blockIdx.y * G::TH;
    const int xi = x0 + tx * DOT_TX + lane, yi = y0 + w;
    const int cx = tx * DOT_TX + lane + 2;  // box column of the own cell
    // planes [zb, ze) in chunks of zc, or with zhi >= 0 the pair of single
    // planes {zb, zhi} (both boundary planes of a slab in one launch)
    const int zs = zhi >= 0 ? (blockIdx.z ? zhi : zb) : zb + blockIdx.z * zc;
    const int zend = zhi >= 0 ? zs + 1 : min(ze, zs + zc);  // zc <= TZC planes per CTA
    const int nzl = g.nzl;
    const bool valid = xi < g.nx && yi < g.ny;
    auto halo = [&](int zl) { return zl < 0 || zl >= nzl; };
    auto stage_of = [&](int zl) { return (int)((unsigned)(zl - zs + 1) % (unsigned)NSTAGE); };
    auto parity_of = [&](int zl) { return ((unsigned)(zl - zs + 1) / (unsigned)NSTAGE) & 1u; };
    auto sa = [&](int zl) { return tsm + stage_of(zl) * G::SA; };
    auto sb = [&](int zl) { return tsm + stage_of(zl) * G::SA + G::BPAD; };
    auto sx = [&](int zl) { return tsm + stage_of(zl) * G::SA + 2 * G::BPAD; };
    // producer: one thread fetches plane zl into its stage
    auto issue = [&](int zl) {
        uint64_t *b = &bar[stage_of(zl)];
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        if (halo(zl)) {
            mbar_expect_tx(b, G::BOX * 8);
            tma_load_3d(sa(zl), &m_pn, b, x0 - 2, y0 - 1, zl + 1);
        } else {
            const bool wx = dox && zl >= zs && zl < zend;
            mbar_expect_tx(b, 2 * G::BOX * 8 + (wx ? G::OWN * 8 : 0));
            tma_load_3d(sa(zl), &m_r, b, x0 - 2, y0 - 1, zl + 1);
            tma_load_3d(sb(zl), &m_po, b, x0 - 2, y0 - 1, zl + 1);
            if (wx) tma_load_3d(sx(zl), &m_x, b, x0, y0, zl + 1);
        }
    };
    if (tid == 0) {
        for (int k = 0; k < NSTAGE; ++k) mbar_init(&bar[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (tid == 0)
        for (int zl = zs - 1; zl <= min(zs + NSTAGE - 2, zend); ++zl) issue(zl);
    // p_new at box cell (yy, xx) of plane zl's stage
    auto U = [&](int zl, int yy, int xx) -> double {
        const int e = yy * G::BXW + xx;
        return halo(zl) ? sa(zl)[e] : fma(beta, sb(zl)[e], sa(zl)[e]);
    };
    mbar_wait(&bar[stage_of(zs - 1)], parity_of(zs - 1));
    mbar_wait(&bar[stage_of(zs)], parity_of(zs));
    double below = U(zs - 1, w + 1, cx);
    double center = U(zs, w + 1, cx);
    const int64_t o = (int64_t)yi * g.pitch + xi + g.ps;  // (xi, yi, zl = 0)
    // The plane loop is unrolled by the ring depth: plane z = zq + k sits in
    // stage (k + 1) % NSTAGE, a compile-time constant, so every shared-memory
    // read is a fixed offset from the ring base.  Planes z in [zs, zend) are
    // inside the slab (never halo); only the plane above may be a halo plane.
    const int c = (w + 1) * G::BXW + cx;  // own cell in a box
    const int cown = 2 * G::BPAD + w * G::TW + cx - 2;  // own cell in the stage's x tile
    const int64_t ps = g.ps;
    double *pnp = DOMAP ? pn + o + (int64_t)zs * g.ps : nullptr;
    double *xsp = dox ? xs + o + (int64_t)zs * g.ps : nullptr;
    double *c1p = C1 ? c1_out + o + (int64_t)zs * g.ps : nullptr;
    for (int zq = zs, q = 0; zq < zend; zq += NSTAGE, ++q) {
        double pv[NSTAGE];  // this group's per-plane row products, reduced together below
#pragma unroll
        for (int k = 0; k < NSTAGE; ++k) {
            const int z = zq + k;
            pv[k] = 0.0;
            if (z >= zend) continue;  // CTA-uniform
            const int s0 = (k + 1) % NSTAGE, s1 = (k + 2) % NSTAGE;  // stages of planes z, z + 1
            if (tid == 0) mbar_wait(&bar[s1], (unsigned)(q + (k + 2) / NSTAGE) & 1u);
            __syncthreads();
            if (tid == 0 && z + NSTAGE - 1 <= zend) issue(z + NSTAGE - 1);  // -> stage k (plane z-1)
            const double *A1 = tsm + s1 * G::SA, *A0 = tsm + s0 * G::SA;
            const double *B1 = A1 + G::BPAD, *B0 = A0 + G::BPAD;
            const double above = z + 1 >= nzl ? A1[c] : fma(beta, B1[c], A1[c]);
            double prod = 0.0;
            if (valid) {
                double s = __dadd_rn(fma(beta, B0[c - 1], A0[c - 1]), fma(beta, B0[c + 1], A0[c + 1]));
                s = __dadd_rn(s, fma(beta, B0[c - G::BXW], A0[c - G::BXW]));
                s = __dadd_rn(s, fma(beta, B0[c + G::BXW], A0[c + G::BXW]));
                s = __dadd_rn(s, below);
                s = __dadd_rn(s, above);
                const double qv = C1 ? fma(-6.0, center, s) : fma(6.0, center, -s);
                if (C1) __stcs(c1p, qv);
                if (DOMAP) {
                    *pnp = center;
                    if (dox) *xsp = fma(ap, B0[c], A0[cown]);
                }
                prod = __dmul_rn(center, qv);
            }
            if (DOMAP) pnp += ps;
            if (dox) xsp += ps;
            if (C1) c1p += ps;
            pv[k] = prod;
            below = center;
            center = above;
        }
        // the NSTAGE row sums of the group in one transposed butterfly (bitwise
        // equal to NSTAGE warp_sum_canon calls, a third of the shuffles)
        const double v = warp_sum_multi<NSTAGE>(pv, lane);
        const int i = warp_multi_index<NSTAGE>(lane);
        if ((lane & (32 / WarpMulti<NSTAGE>::M - 1)) == 0 && i < NSTAGE && zq + i < zend) sw[zq + i - zs][t][wr] = v;
    }
    __syncthreads();  // sw complete
    // per-plane tile partials: the 8 row values in increasing y
    if (tid < (zend - zs) * NTX * NTY) {
        const int zi = tid / (NTX * NTY), tt = tid % (NTX * NTY);
        const int tile_x = blockIdx.x * NTX + tt % NTX, tile_y = blockIdx.y * NTY + tt / NTX;
        double s = sw[zi][tt][0];
#pragma unroll
        for (int k = 1; k < DOT_TY; ++k) s = __dadd_rn(s, sw[zi][tt][k]);
        if (tile_x < tiles_x && tile_y * DOT_TY < g.ny)
            tp[((int64_t)g.z0 + zs + zi) * T + (int64_t)tile_y * tiles_x + tile_x] = s;
    }
    pdl_trigger();  // this CTA's results are stored: the next kernel may launch
}

// ---------------------------------------------------------------------------
// CG phase B, TMA-staged: q = A p_new from the stored p_new ((32 NTX + 4) x
// 10 box per plane, halo planes included), r -= alpha q (own box of r per
// plane), per-plane tile partial of r*r in the ZR = 1 canonical order
// (butterfly per row, rows in increasing y).
// ---------------------------------------------------------------------------
template <class G>
__global__ void __launch_bounds__(G::NT, G::MINB_B)
    k_cgB_tma(const __grid_constant__ CUtensorMap m_p, const __grid_constant__ CUtensorMap m_r, double *r, PGeo g,
              int zb, int ze, const CgScal *sc, double *tp, int T, int tiles_x, int zc) {
    constexpr int NTX = G::TW / DOT_TX, NTY = G::TH / DOT_TY, NSTAGE = G::NST;
    extern __shared__ __align__(128) double tsm[];
    __shared__ __align__(8) uint64_t bar[NSTAGE];
    __shared__ double sw[TZC][NTY * NTX][DOT_TY];
    pdl_wait();
    if (sc->status != 0) return;
    const double alpha = sc->alpha;
    // warp -> (dot tile t = (ty, tx) of the CTA, row wr of that tile); w = CTA row
    const int tid = threadIdx.x, lane = tid & 31, wr = (tid >> 5) % DOT_TY, t = (tid >> 5) / DOT_TY;
    const int tx = t % NTX, ty = t / NTX, w = ty * DOT_TY + wr;
    const int x0 = blockIdx.x * G::TW, y0 = blockIdx.y * G::TH;
    const int xi = x0 + tx * DOT_TX + lane, yi = y0 + w;
    const int cx = tx * DOT_TX + lane + 2;
    const int zs = zb + blockIdx.z * zc, zend = min(ze, zs + zc);
    const bool valid = xi < g.nx && yi < g.ny;
    auto stage_of = [&](int zl) { return (int)((unsigned)(zl - zs + 1) % (unsigned)NSTAGE); };
    auto parity_of = [&](int zl) { return ((unsigned)(zl - zs + 1) / (unsigned)NSTAGE) & 1u; };
    auto sp = [&](int zl) { return tsm + stage_of(zl) * G::SB; };
    auto sr = [&](int zl) { return tsm + stage_of(zl) * G::SB + G::BPAD; };
    auto issue = [&](int zl) {
        uint64_t *b = &bar[stage_of(zl)];
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        const bool wr = zl >= zs && zl < zend;
        mbar_expect_tx(b, G::BOX * 8 + (wr ? G::OWN * 8 : 0));
        tma_load_3d(sp(zl), &m_p, b, x0 - 2, y0 - 1, zl + 1);
        if (wr) tma_load_3d(sr(zl), &m_r, b, x0, y0, zl + 1);
    };
    if (tid == 0) {
        for (int k = 0; k < NSTAGE; ++k) mbar_init(&bar[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (tid == 0)
        for (int zl = zs - 1; zl <= min(zs + NSTAGE - 2, zend); ++zl) issue(zl);
    mbar_wait(&bar[stage_of(zs - 1)], parity_of(zs - 1));
    mbar_wait(&bar[stage_of(zs)], parity_of(zs));
    const int c = (w + 1) * G::BXW + cx;
    double below = sp(zs - 1)[c];
    double center = sp(zs)[c];
    const int64_t o = (int64_t)yi * g.pitch + xi + g.ps;
    double *rp = r + o + (int64_t)zs * g.ps;
    const int cown = G::BPAD + w * G::TW + cx - 2;  // own cell in the stage's r tile
    const int64_t ps = g.ps;
    for (int zq = zs, q = 0; zq < zend; zq += NSTAGE, ++q) {
        double pv[NSTAGE];  // this group's per-plane row products, reduced together below
#pragma unroll
        for (int k = 0; k < NSTAGE; ++k) {
            const int z = zq + k;
            pv[k] = 0.0;
            if (z >= zend) continue;  // CTA-uniform
            const int s0 = (k + 1) % NSTAGE, s1 = (k + 2) % NSTAGE;  // stages of planes z, z + 1
            if (tid == 0) mbar_wait(&bar[s1], (unsigned)(q + (k + 2) / NSTAGE) & 1u);
            __syncthreads();
            if (tid == 0 && z + NSTAGE - 1 <= zend) issue(z + NSTAGE - 1);  // -> stage k (plane z-1)
            const double *pz = tsm + s0 * G::SB;
            const double above = (tsm + s1 * G::SB)[c];
            double prod = 0.0;
            if (valid) {
                double s = __dadd_rn(pz[c - 1], pz[c + 1]);
                s = __dadd_rn(s, pz[c - G::BXW]);
                s = __dadd_rn(s, pz[c + G::BXW]);
                s = __dadd_rn(s, below);
                s = __dadd_rn(s, above);
                const double qv = fma(6.0, center, -s);
                const double rn = fma(-alpha, qv, pz[cown]);
                __stcs(rp, rn);
                prod = __dmul_rn(rn, rn);
            }
            rp += ps;
            pv[k] = prod;
            below = center;
            center = above;
        }
        // the NSTAGE row sums of the group in one transposed butterfly (bitwise
        // equal to NSTAGE warp_sum_canon calls, a third of the shuffles)
        const double v = warp_sum_multi<NSTAGE>(pv, lane);
        const int i = warp_multi_index<NSTAGE>(lane);
        if ((lane & (32 / WarpMulti<NSTAGE>::M - 1)) == 0 && i < NSTAGE && zq + i < zend) sw[zq + i - zs][t][wr] = v;
    }
    __syncthreads();
    if (tid < (zend - zs) * NTX * NTY) {
        const int zi = tid / (NTX * NTY), tt = tid % (NTX * NTY);
        const int tile_x = blockIdx.x * NTX + tt % NTX, tile_y = blockIdx.y * NTY + tt / NTX;
        double s = sw[zi][tt][0];
#pragma unroll
        for (int k = 1; k < DOT_TY; ++k) s = __dadd_rn(s, sw[zi][tt][k]);
        if (tile_x < tiles_x && tile_y * DOT_TY < g.ny)
            tp[((int64_t)g.z0 + zs + zi) * T + (int64_t)tile_y * tiles_x + tile_x] = s;
    }
    pdl_trigger();  // this CTA's results are stored: the next kernel may launch
}

// ---------------------------------------------------------------------------
// host side: tensor maps (cached per buffer and geometry)
// ---------------------------------------------------------------------------
// planes per CTA.  Every CTA marches zc planes (plus ~H planes of set-up:
// the two z-halo planes of the ring and the first load's latency), so a
// launch costs about ceil(CTAs / resident CTAs) x (zc + H).  zc is the
// power-of-two divisor of TZC (down to 2) that minimises that estimate:
// 512^3 on one GPU keeps 32 (19 waves of 444 CTAs); a 64-plane slab (512^3
// on 8 GPUs) takes 16 (5 waves instead of 3 partly empty ones).  The dot
// partials are per plane and tile, so results do not depend on zc.
// NB_CG_ZC=<n> forces n.
static int sm_count() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
    }
    return n;
}
static int tma_zc(int ctas_per_plane, int nplanes, int ctas_per_sm) {
    static int forced = -1;
    if (forced < 0) forced = getenv("NB_CG_ZC") ? std::max(1, std::min(TZC, atoi(getenv("NB_CG_ZC")))) : 0;
    if (forced) return forced;
    static std::mutex mu;
    static std::map<std::tuple<int, int, int>, int> cache;
    std::lock_guard<std::mutex> lk(mu);
    const auto key = std::make_tuple(ctas_per_plane, nplanes, ctas_per_sm);
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    // every zc in [2, TZC]: CTAs are dispatched in launch order (the chunks
    // of a plane range one after another, the last one possibly shorter)
    // onto cap resident slots; a CTA of p planes costs p + H plane-times
    // (H: the ring's two z-halo planes and the first load's latency).  The
    // simulated makespan picks zc (non-powers of two cut the last wave's
    // idle slots: 62 planes at 512 CTAs per plane take 13, not 16)
    const int cap = std::max(1, sm_count() * ctas_per_sm);
    constexpr double H = 3.0;
    int best = TZC;
    double best_cost = 1e300;
    std::vector<double> slot;
    static const bool pow2 = getenv("NB_CG_ZC_POW2") != nullptr;  // the round-1 search (powers of two)
    for (int zc = TZC; zc >= 2; zc = pow2 ? zc / 2 : zc - 1) {
        const int nchunk = (nplanes + zc - 1) / zc;
        slot.assign(cap, 0.0);
        std::priority_queue<double, std::vector<double>, std::greater<double>> free_at(slot.begin(), slot.end());
        double end = 0.0;
        for (int c = 0; c < nchunk; ++c) {
            const double dur = std::min(zc, nplanes - c * zc) + H;
            for (int k = 0; k < ctas_per_plane; ++k) {
                const double t0 = free_at.top();
                free_at.pop();
                free_at.push(t0 + dur);
                end = std::max(end, t0 + dur);
            }
        }
        if (end < best_cost - 1e-9) best_cost = end, best = zc;
    }
    cache[key] = best;
    return best;
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

// tensor map of a partition buffer with a bw x bh x 1 box (cached)
nb_status tmap_box(const void *base, const PGeo &g, int bw, int bh, CUtensorMap *out) {
    std::lock_guard<std::mutex> lk(g_tmap_mu);
    auto key = std::make_tuple(base, g.nx, g.ny, g.nzl, g.pitch, bw * 1024 + bh);
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
    cuuint32_t boxd[3] = {(cuuint32_t)bw, (cuuint32_t)bh, 1};
    cuuint32_t es[3] = {1, 1, 1};
    CUresult r = fn(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, const_cast<void *>(base), dims, strides, boxd, es,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) NB_FAIL(NB_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
    g_tmaps[key] = m;
    *out = m;
    return NB_OK;
}

// box: 0 = (tile + ring) 36 x 10 x 1 (x from x0-2), 1 = own tile 32 x 8 x 1
nb_status tmap_for(const void *base, const PGeo &g, int box, CUtensorMap *out) {
    return box == 0 ? tmap_box(base, g, DOT_TX + 4, DOT_TY + 2, out) : tmap_box(base, g, DOT_TX, DOT_TY, out);
}

// drop cached maps whose base lies in [lo, hi) (a freed or unwrapped buffer)
void nb_tma_forget_range(const void *lo, const void *hi) {
    std::lock_guard<std::mutex> lk(g_tmap_mu);
    for (auto it = g_tmaps.begin(); it != g_tmaps.end();) {
        const char *b = (const char *)std::get<0>(it->first);
        it = (b >= (const char *)lo && b < (const char *)hi) ? g_tmaps.erase(it) : std::next(it);
    }
}

bool nb_tma_enabled() {
    static int en = -1;
    if (en < 0) en = getenv("NB_NO_TMA") ? 0 : 1;
    return en && encode_fn() != nullptr;
}

// dynamic shared memory of the ring (set once per kernel instantiation)
template <class F>
static void tma_smem_attr(F *f, int bytes) {
    static std::mutex mu;
    static std::map<const void *, int> done;
    std::lock_guard<std::mutex> lk(mu);
    if (done[(const void *)f] < bytes) {
        cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
        done[(const void *)f] = bytes;
    }
}

template <bool DOMAP, bool C1, class G>
static nb_status launch_cgA(nb_grid *g, const PGeo &geo, const double *r, const double *po, double *pn, double *x,
                            int zb, int ze, const CgScal *sc, double c1_a, double *c1_out, const char *label,
                            int zhi = -1) {
    CUtensorMap mr, mpo, mpn, mx;
    NB_TRY(tmap_box(r, geo, G::BXW, G::BYH, &mr));
    NB_TRY(tmap_box(po, geo, G::BXW, G::BYH, &mpo));
    NB_TRY(tmap_box(pn, geo, G::BXW, G::BYH, &mpn));
    NB_TRY(tmap_box(C1 ? r : x, geo, C1 ? G::BXW : G::TW, C1 ? G::BYH : G::TH, &mx));
    constexpr int NTX = G::TW / DOT_TX, NTY = G::TH / DOT_TY;
    const int zc = tma_zc(((g->tiles_x + NTX - 1) / NTX) * ((g->tiles_y + NTY - 1) / NTY), ze - zb, G::MINB_A);
    const int smem = G::NST * G::SA * 8;
    tma_smem_attr(k_cgA_tma<DOMAP, C1, G>, smem);
    dim3 blk(G::NT),
        grd((g->tiles_x + NTX - 1) / NTX, (g->tiles_y + NTY - 1) / NTY, zhi >= 0 ? 2 : (ze - zb + zc - 1) / zc);
    LaunchScope ls(g, g->cs, label);
    NB_CUDA(nb_launch_ex(k_cgA_tma<DOMAP, C1, G>, grd, blk, (size_t)smem, g->cs, true, mr, mpo, mpn, mx, pn, x, geo,
                         zb, ze, sc, g->tp, g->T, (int)g->tiles_x, zc, c1_a, c1_out, zhi));
    return nb_launch_check(label);
}

// CG phase A on planes [zb, ze) of a partition (r, p_old, p_new, x buffers)
nb_status nb_cgA_tma(nb_grid *g, const PGeo &geo, const double *r, const double *po, double *pn, double *x, bool domap,
                     int zb, int ze, const CgScal *sc, int zhi) {
    if (ze <= zb) return NB_OK;
    return domap ? launch_cgA<true, false, CgGeo>(g, geo, r, po, pn, x, zb, ze, sc, 0.0, nullptr, "k_msr_cgA", zhi)
                 : launch_cgA<false, false, CgGeo>(g, geo, r, po, pn, x, zb, ze, sc, 0.0, nullptr, "k_msr_cgA", zhi);
}

// C1 map-stencil-reduce on planes [zb, ze): x_out = x_in + a y_in (stored
// when domap), y_out = L(x_out), per-plane tile partials of x_out * y_out
nb_status nb_c1_tma(nb_grid *g, const PGeo &geo, const double *xin, const double *yin, double *xout, double *yout,
                    double a, bool domap, int zb, int ze, int zhi) {
    if (ze <= zb) return NB_OK;
    return domap ? launch_cgA<true, true, CgGeo>(g, geo, xin, yin, xout, nullptr, zb, ze, nullptr, a, yout, "k_msr_c1",
                                                 zhi)
                 : launch_cgA<false, true, CgGeo>(g, geo, xin, yin, xout, nullptr, zb, ze, nullptr, a, yout, "k_msr_c1",
                                                  zhi);
}

// CG phase B on planes [zb, ze) of a partition (stored p_new, r)
nb_status nb_cgB_tma(nb_grid *g, const PGeo &geo, const double *p, double *r, int zb, int ze, const CgScal *sc) {
    if (ze <= zb) return NB_OK;
    using G = CgGeo;
    CUtensorMap mp, mr;
    NB_TRY(tmap_box(p, geo, G::BXW, G::BYH, &mp));
    NB_TRY(tmap_box(r, geo, G::TW, G::TH, &mr));
    constexpr int NTX = G::TW / DOT_TX, NTY = G::TH / DOT_TY;
    const int zc = tma_zc(((g->tiles_x + NTX - 1) / NTX) * ((g->tiles_y + NTY - 1) / NTY), ze - zb, G::MINB_B);
    const int smem = G::NST * G::SB * 8;
    tma_smem_attr(k_cgB_tma<G>, smem);
    dim3 blk(G::NT), grd((g->tiles_x + NTX - 1) / NTX, (g->tiles_y + NTY - 1) / NTY, (ze - zb + zc - 1) / zc);
    LaunchScope ls(g, g->cs, "k_cg_B");
    NB_CUDA(nb_launch_ex(k_cgB_tma<G>, grd, blk, (size_t)smem, g->cs, true, mp, mr, r, geo, zb, ze, sc, g->tp, g->T,
                         (int)g->tiles_x, zc));
    return nb_launch_check("k_cgB_tma");
}
