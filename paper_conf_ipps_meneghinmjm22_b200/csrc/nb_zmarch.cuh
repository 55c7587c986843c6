// nb_zmarch.cuh — the z-march skeleton shared by every dense 7-point kernel.
//
// A CTA of 8 warps owns a 32 x (8*ZR) xy tile and marches ZC planes up the
// slab.  Lane = x; warp w owns the ZR consecutive rows y0 + w*ZR + j, so each
// thread updates ZR cells per plane with ZR independent loads in flight per
// array.  Each thread keeps the z-1 / z / z+1 values of its cells in
// registers.  x/y neighbours:
//   SMEM = false: y within the thread from registers; x and the rows across
//                 warp edges by direct loads (L1 hits); no barriers.
//   SMEM = true : the stencil input is itself computed (the CG / C1 map output
//                 recomputed from its operands), so the plane tile plus a
//                 one-cell ring is staged once per plane in a double-buffered
//                 shared tile; the ring's raw loads are issued together with
//                 the own cells'.  One barrier per plane.
//
// Canonical dot order per plane and 32 x 8 dot tile: per lane
// the ZR rows of a warp in increasing y (sequential adds), xor-butterfly over
// the 32 lanes, then the 8/ZR warps of the tile in increasing y.  Standalone
// nb_dot (k_dot) follows the same order, so fused and standalone dots of the
// same data agree bit for bit.
//
// The Op supplies:
//   T, Raw                      stencil value type; raw per-cell loads
//   static constexpr bool DOT   whether a dot contribution is produced
//   bool skip(); void init()    uniform early exit; device scalars
//   T outside()                 value of out-of-domain x/y neighbours
//   Raw raw(int zl, int64_t i, bool own)  issue the loads of cell i on plane
//                               zl (own: also the epilogue's operands)
//   T val(int zl, const Raw&)   stencil input from the raw loads
//   T nval(int zl, int64_t i)   stencil input of a neighbour (load + val)
//   double cell(int zl, int64_t i, T c, T s, const Raw &rc)   epilogue with
//        the canonical neighbour sum s = ((((xm+xp)+ym)+yp)+zm)+zp and the
//        centre's raw loads; returns the dot contribution (0 if !DOT)
#pragma once
#include "nb_device.cuh"

// Rows per thread: ZR_MAP for the kernels whose stencil input is a
// recomputed map output (CG phase A, C1: shared-memory staging), ZR_STO for
// the kernels reading a stored input (CG phase B / set-up, Laplacian, dot).
// The canonical order of a dot depends on ZR, so every kernel producing the
// same dot uses the same ZR (phase A's <p,q> in all OCC variants: ZR_MAP;
// <r,r> and nb_dot: ZR_STO).
#ifndef NB_ZR_MAP
#define NB_ZR_MAP 1
#endif
#ifndef NB_ZR_STO
#define NB_ZR_STO 1
#endif
#ifndef NB_ZC
#define NB_ZC 32
#endif
constexpr int ZC = NB_ZC;               // planes per CTA
constexpr int ZW = 8;                   // warps per CTA
constexpr int ZR_MAP = NB_ZR_MAP, ZR_STO = NB_ZR_STO;
static_assert(DOT_TY % ZR_MAP == 0 && DOT_TY % ZR_STO == 0, "ZR must divide the dot tile height");

template <typename T>
__device__ __forceinline__ T add_rn(T a, T b);
template <>
__device__ __forceinline__ double add_rn<double>(double a, double b) { return __dadd_rn(a, b); }
template <>
__device__ __forceinline__ float add_rn<float>(float a, float b) { return __fadd_rn(a, b); }

// the per-plane warp partials of a chunk -> canonical dot-tile values
template <int ZR>
__device__ __forceinline__ void zm_flush(const double (&sw)[ZC][ZW], int nplanes, double *tp, int64_t pbase, int T,
                                         int tiles_x, int tiles_y, int bx, int by) {
    constexpr int WPT = DOT_TY / ZR;  // warps per canonical dot tile
    const int t = threadIdx.x;
    if (t < nplanes * ZR) {
        const int zi = t / ZR, k = t % ZR;  // k-th dot tile of the CTA
        const int tile_y = by * ZR + k;
        if (tile_y < tiles_y) {
            double s = sw[zi][k * WPT];
#pragma unroll
            for (int w = 1; w < WPT; ++w) s = __dadd_rn(s, sw[zi][k * WPT + w]);
            tp[(pbase + zi) * (int64_t)T + tile_y * tiles_x + bx] = s;
        }
    }
}

// L = lookahead: 0 loads plane z+1 at step z; 1 prefetches plane z+2 at step
// z (own cells and ring), so the barrier never waits on DRAM latency
template <class Op, bool SMEM, int L, int ZR>
__global__ void __launch_bounds__(32 * ZW) k_zmarch(Op op, PGeo g, int zb, int ze, double *tp, int T, int tiles_y) {
    constexpr int ZTY = ZW * ZR;  // CTA tile rows
    using V = typename Op::T;
    using Raw = typename Op::Raw;
    __shared__ V sU[SMEM ? 2 : 1][SMEM ? ZTY + 2 : 1][DOT_TX + 2];
    __shared__ double sw[ZC][ZW];
    if (op.skip()) return;
    op.init();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int x0 = blockIdx.x * DOT_TX, y0 = blockIdx.y * ZTY;
    const int xi = x0 + lane, yr = y0 + w * ZR;
    const int zs = zb + blockIdx.z * ZC, zend = min(ze, zs + ZC);
    const bool xin = xi < g.nx;
    const V out = op.outside();
    const int64_t o0 = (int64_t)yr * g.pitch + xi + g.ps;  // (xi, yr, zl = 0)
    auto in = [&](int j) { return xin && yr + j < g.ny; };
    auto idx = [&](int xx, int yy, int zl) { return (int64_t)(zl + 1) * g.ps + (int64_t)yy * g.pitch + xx; };
    // ring roles (SMEM): warp 0 -> row y0-1, warp ZW-1 -> row y0+ZTY,
    // lane 0 -> column x0-1 of the warp's rows, lane 31 -> column x0+32
    const bool rrow = SMEM && (w == 0 || w == ZW - 1);
    const int ry = w == 0 ? y0 - 1 : y0 + ZTY;
    const bool rrow_in = rrow && xin && ry >= 0 && ry < g.ny;
    const bool rcol = SMEM && (lane == 0 || lane == 31);
    const int rx = lane == 0 ? x0 - 1 : x0 + DOT_TX;
    const bool rcol_x = rcol && rx >= 0 && rx < g.nx;
    auto ring_store = [&](int b, int zl, const Raw &qr, const Raw (&qc)[ZR]) {
        if (rrow) sU[b][w == 0 ? 0 : ZTY + 1][lane + 1] = rrow_in ? op.val(zl, qr) : out;
        if (rcol) {
#pragma unroll
            for (int j = 0; j < ZR; ++j)
                sU[b][w * ZR + j + 1][lane == 0 ? 0 : DOT_TX + 1] =
                    (rcol_x && yr + j < g.ny) ? op.val(zl, qc[j]) : out;
        }
    };
    auto ring_load = [&](int zl, Raw &qr, Raw (&qc)[ZR]) {
        if (rrow_in) qr = op.raw(zl, idx(xi, ry, zl), false);
        if (rcol_x) {
#pragma unroll
            for (int j = 0; j < ZR; ++j)
                if (yr + j < g.ny) qc[j] = op.raw(zl, idx(rx, yr + j, zl), false);
        }
    };
    V below[ZR], center[ZR], above[ZR];
    Raw rc[ZR], ra[ZR], rb[ZR];
    Raw gr{}, gc[ZR], gr2{}, gc2[ZR];
#pragma unroll
    for (int j = 0; j < ZR; ++j) {
        below[j] = center[j] = out;
        rc[j] = ra[j] = rb[j] = gc[j] = gc2[j] = Raw{};
        if (in(j)) {
            const int64_t i = o0 + (int64_t)j * g.pitch;
            below[j] = op.val(zs - 1, op.raw(zs - 1, i + (int64_t)(zs - 1) * g.ps, false));
            rc[j] = op.raw(zs, i + (int64_t)zs * g.ps, true);
            if (L == 1) ra[j] = op.raw(zs + 1, i + (int64_t)(zs + 1) * g.ps, true);
        }
    }
    if (SMEM) ring_load(zs, gr, gc);
    if (SMEM && L == 1 && zs + 1 < zend) ring_load(zs + 1, gr2, gc2);
#pragma unroll
    for (int j = 0; j < ZR; ++j)
        if (in(j)) center[j] = op.val(zs, rc[j]);
    if (SMEM) {
#pragma unroll
        for (int j = 0; j < ZR; ++j) sU[0][w * ZR + j + 1][lane + 1] = center[j];
        ring_store(0, zs, gr, gc);
    }
    for (int z = zs; z < zend; ++z) {
        const int b = SMEM ? ((z - zs) & 1) : 0;
        const int64_t ic = o0 + (int64_t)z * g.ps;
        // loads of the step: L = 0: plane z+1 now; L = 1: plane z+2 (plane
        // z+1 arrived during the previous step)
        if (L == 0) {
#pragma unroll
            for (int j = 0; j < ZR; ++j)
                if (in(j)) ra[j] = op.raw(z + 1, ic + (int64_t)j * g.pitch + g.ps, true);
            if (SMEM && z + 1 < zend) ring_load(z + 1, gr, gc);
        } else {
#pragma unroll
            for (int j = 0; j < ZR; ++j)
                if (in(j) && z + 2 <= zend) rb[j] = op.raw(z + 2, ic + (int64_t)j * g.pitch + 2 * g.ps, true);
            if (SMEM && z + 2 < zend) ring_load(z + 2, gr, gc);
        }
#pragma unroll
        for (int j = 0; j < ZR; ++j) above[j] = in(j) ? op.val(z + 1, ra[j]) : out;
        if (SMEM) __syncthreads();
        double col = 0.0;
#pragma unroll
        for (int j = 0; j < ZR; ++j) {
            double prod = 0.0;
            if (in(j)) {
                const int64_t i = ic + (int64_t)j * g.pitch;
                const int y = yr + j;
                V xm, xp, ym, yp;
                if (SMEM) {
                    xm = sU[b][w * ZR + j + 1][lane];
                    xp = sU[b][w * ZR + j + 1][lane + 2];
                    ym = sU[b][w * ZR + j][lane + 1];
                    yp = sU[b][w * ZR + j + 2][lane + 1];
                } else {
                    xm = xi > 0 ? op.nval(z, i - 1) : out;
                    xp = xi < g.nx - 1 ? op.nval(z, i + 1) : out;
                    ym = j > 0 ? center[j - 1] : (y > 0 ? op.nval(z, i - g.pitch) : out);
                    yp = j < ZR - 1 ? center[j + 1] : (y < g.ny - 1 ? op.nval(z, i + g.pitch) : out);
                }
                V s = add_rn<V>(xm, xp);
                s = add_rn<V>(s, ym);
                s = add_rn<V>(s, yp);
                s = add_rn<V>(s, below[j]);
                s = add_rn<V>(s, above[j]);
                prod = op.cell(z, i, center[j], s, rc[j]);
            }
            col = j == 0 ? prod : __dadd_rn(col, prod);
        }
        if (Op::DOT) {
            col = warp_sum_canon(col);
            if (lane == 0) sw[z - zs][w] = col;
        }
        if (SMEM && z + 1 < zend) {
#pragma unroll
            for (int j = 0; j < ZR; ++j) sU[b ^ 1][w * ZR + j + 1][lane + 1] = above[j];
            if (L == 0)
                ring_store(b ^ 1, z + 1, gr, gc);
            else
                ring_store(b ^ 1, z + 1, gr2, gc2);
        }
#pragma unroll
        for (int j = 0; j < ZR; ++j) {
            below[j] = center[j];
            center[j] = above[j];
            rc[j] = ra[j];
            if (L == 1) ra[j] = rb[j];
        }
        if (SMEM && L == 1) {
            gr2 = gr;
#pragma unroll
            for (int j = 0; j < ZR; ++j) gc2[j] = gc[j];
        }
    }
    if (Op::DOT) {
        __syncthreads();
        zm_flush<ZR>(sw, zend - zs, tp, (int64_t)g.z0 + zs, T, gridDim.x, tiles_y, blockIdx.x, blockIdx.y);
    }
}
