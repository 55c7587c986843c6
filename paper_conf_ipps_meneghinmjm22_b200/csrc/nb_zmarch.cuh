// nb_zmarch.cuh — the z-march skeleton shared by every dense 7-point kernel.
//
// A CTA of DOT_TX x DOT_TY threads (warp = one x-row) owns one xy tile and
// marches ZC planes up the slab.  Each thread keeps the z-1 / z / z+1 values
// of its column in registers and PREFETCHES the raw loads of plane z+2 while
// plane z is computed, so every thread always has the next plane's DRAM
// loads in flight.  x/y neighbours:
//   SMEM = false: direct loads (L1 hits: the plane was loaded by the
//                 neighbouring threads of the CTA one iteration earlier);
//                 no barriers at all.
//   SMEM = true : the plane tile plus a one-cell ring is staged in a
//                 double-buffered shared tile (used when the stencil input is
//                 itself computed — the CG/C1 recompute of the map output —
//                 so that every cell's value is computed once); the ring is
//                 prefetched like the own column.  One barrier per plane.
//
// The dot contribution of every plane follows the canonical tile order of
// xor-butterfly over the 32 lanes of a
// row, then the DOT_TY rows in increasing y.
//
// The Op supplies:
//   T, Raw                      stencil value type; raw per-cell loads
//   static constexpr bool DOT   whether a dot contribution is produced
//   bool skip(); void init()    uniform early exit; device scalars
//   T outside()                 value of out-of-domain x/y neighbours
//   Raw raw(int zl, int64_t i)  issue the loads of cell i on plane zl
//   T val(int zl, const Raw&)   stencil input from the raw loads
//   T nval(int zl, int64_t i)   stencil input of a neighbour (load + val)
//   double cell(int zl, int64_t i, T c, T s, const Raw &rc)   epilogue with
//        the canonical neighbour sum s = ((((xm+xp)+ym)+yp)+zm)+zp and the
//        centre's raw loads; returns the dot contribution (0 if !DOT)
#pragma once
#include "nb_device.cuh"

constexpr int ZC = 32;  // planes per CTA

template <typename T>
__device__ __forceinline__ T add_rn(T a, T b);
template <>
__device__ __forceinline__ double add_rn<double>(double a, double b) { return __dadd_rn(a, b); }
template <>
__device__ __forceinline__ float add_rn<float>(float a, float b) { return __fadd_rn(a, b); }

template <class Op, bool SMEM, int L>
__global__ void __launch_bounds__(DOT_TX *DOT_TY) k_zmarch(Op op, PGeo g, int zb, int ze, double *tp, int T) {
    using V = typename Op::T;
    using Raw = typename Op::Raw;
    __shared__ V sU[SMEM ? 2 : 1][DOT_TY + 2][DOT_TX + 2];
    __shared__ TileStage<ZC> st;
    if (op.skip()) return;
    op.init();
    const int tx = threadIdx.x, ty = threadIdx.y;
    const int x0 = blockIdx.x * DOT_TX, y0 = blockIdx.y * DOT_TY;
    const int xi = x0 + tx, yi = y0 + ty;
    const int zs = zb + blockIdx.z * ZC, zend = min(ze, zs + ZC);
    const bool valid = xi < g.nx && yi < g.ny;
    const V out = op.outside();
    const int64_t o = (int64_t)(valid ? yi : 0) * g.pitch + (valid ? xi : 0) + g.ps;  // (xi, yi, zl = 0)
    // ring cell of this thread (SMEM): at most one per thread except corners
    // — rows y0-1 / y0+TY by warps 0 / TY-1, columns x0-1 / x0+TX by lanes 0 / 31
    bool has0 = false, has1 = false;  // this thread fills a ring row / ring column cell
    int rx0 = 0, ry0 = 0, rx1 = 0, ry1 = 0;
    if (SMEM) {
        if (ty == 0) { has0 = true; rx0 = xi; ry0 = y0 - 1; }
        if (ty == DOT_TY - 1) { has0 = true; rx0 = xi; ry0 = y0 + DOT_TY; }
        if (tx == 0) { has1 = true; rx1 = x0 - 1; ry1 = yi; }
        if (tx == DOT_TX - 1) { has1 = true; rx1 = x0 + DOT_TX; ry1 = yi; }
    }
    const bool r0in = has0 && rx0 >= 0 && rx0 < g.nx && ry0 >= 0 && ry0 < g.ny;
    const bool r1in = has1 && rx1 >= 0 && rx1 < g.nx && ry1 >= 0 && ry1 < g.ny;
    const int64_t ro0 = r0in ? (int64_t)ry0 * g.pitch + rx0 + g.ps : 0;
    const int64_t ro1 = r1in ? (int64_t)ry1 * g.pitch + rx1 + g.ps : 0;
    auto ring_store = [&](int b, int zl, const Raw &q0, const Raw &q1) {
        if (!SMEM) return;
        if (has0) sU[b][ty == 0 ? 0 : DOT_TY + 1][tx + 1] = r0in ? op.val(zl, q0) : out;
        if (has1) sU[b][ty + 1][tx == 0 ? 0 : DOT_TX + 1] = r1in ? op.val(zl, q1) : out;
    };
    Raw rc{}, r1{}, r2{}, g0c{}, g0n{}, g1c{}, g1n{};
    V below = out, center = out;
    if (valid) {
        below = op.val(zs - 1, op.raw(zs - 1, o + (int64_t)(zs - 1) * g.ps, false));
        rc = op.raw(zs, o + (int64_t)zs * g.ps, true);
        if (L == 1) r1 = op.raw(zs + 1, o + (int64_t)(zs + 1) * g.ps, true);
    }
    if (r0in) g0c = op.raw(zs, ro0 + (int64_t)(zs) * g.ps, false);
    if (r1in) g1c = op.raw(zs, ro1 + (int64_t)(zs) * g.ps, false);
    if (L == 1 && r0in && zs + 1 < zend) g0n = op.raw(zs + 1, ro0 + (int64_t)(zs + 1) * g.ps, false);
    if (L == 1 && r1in && zs + 1 < zend) g1n = op.raw(zs + 1, ro1 + (int64_t)(zs + 1) * g.ps, false);
    if (valid) center = op.val(zs, rc);
    if (SMEM) {
        sU[0][ty + 1][tx + 1] = center;
        ring_store(0, zs, g0c, g1c);
    }
    for (int z = zs; z < zend; ++z) {
        const int b = SMEM ? ((z - zs) & 1) : 0;
        const int64_t ic = o + (int64_t)z * g.ps;
        // L = 1: prefetch plane z+2 (own column and ring) while plane z is
        // computed; L = 0: load plane z+1 now
        Raw g0f{}, g1f{};
        if (L == 1) {
            if (valid && z + 2 <= zend) r2 = op.raw(z + 2, ic + 2 * g.ps, true);
            if (r0in && z + 2 < zend) g0f = op.raw(z + 2, ro0 + (int64_t)(z + 2) * g.ps, false);
            if (r1in && z + 2 < zend) g1f = op.raw(z + 2, ro1 + (int64_t)(z + 2) * g.ps, false);
        } else {
            if (valid) r1 = op.raw(z + 1, ic + g.ps, true);
            if (r0in && z + 1 < zend) g0n = op.raw(z + 1, ro0 + (int64_t)(z + 1) * g.ps, false);
            if (r1in && z + 1 < zend) g1n = op.raw(z + 1, ro1 + (int64_t)(z + 1) * g.ps, false);
        }
        const V above = valid ? op.val(z + 1, r1) : out;
        if (SMEM) __syncthreads();
        double prod = 0.0;
        if (valid) {
            V xm, xp, ym, yp;
            if (SMEM) {
                xm = sU[b][ty + 1][tx];
                xp = sU[b][ty + 1][tx + 2];
                ym = sU[b][ty][tx + 1];
                yp = sU[b][ty + 2][tx + 1];
            } else {
                xm = xi > 0 ? op.nval(z, ic - 1) : out;
                xp = xi < g.nx - 1 ? op.nval(z, ic + 1) : out;
                ym = yi > 0 ? op.nval(z, ic - g.pitch) : out;
                yp = yi < g.ny - 1 ? op.nval(z, ic + g.pitch) : out;
            }
            V s = add_rn<V>(xm, xp);
            s = add_rn<V>(s, ym);
            s = add_rn<V>(s, yp);
            s = add_rn<V>(s, below);
            s = add_rn<V>(s, above);
            prod = op.cell(z, ic, center, s, rc);
        }
        if (Op::DOT) tile_stage_put<ZC>(st, z - zs, prod);
        if (SMEM && z + 1 < zend) {
            sU[b ^ 1][ty + 1][tx + 1] = above;
            ring_store(b ^ 1, z + 1, g0n, g1n);
        }
        below = center;
        center = above;
        rc = r1;
        if (L == 1) {
            r1 = r2;
            g0n = g0f;
            g1n = g1f;
        }
    }
    if (Op::DOT) {
        __syncthreads();
        tile_stage_flush<ZC>(st, zend - zs, tp, (int64_t)g.z0 + zs, T, blockIdx.y * gridDim.x + blockIdx.x);
    }
}
