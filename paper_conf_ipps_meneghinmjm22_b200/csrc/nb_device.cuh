// nb_device.cuh — device helpers shared by the kernels of libnb.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

#include "nb_internal.cuh"

// Bulk L2 prefetch of [p, p + bytes) (p 16-byte aligned, bytes a multiple
// of 16): the copy engine of the SM fetches the lines into L2 without
// holding a register or a thread; a later load of them is an L2 hit.
__device__ __forceinline__ void nb_prefetch_l2(const void *p, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

// xor-butterfly warp sum (offsets 16, 8, 4, 2, 1).  IEEE addition is
// commutative, so every lane ends with the same bits: the value is a fixed
// function of the 32 inputs.
__device__ __forceinline__ double warp_sum_canon(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = __dadd_rn(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

// N canonical warp sums at once (transposed butterfly).  Bitwise equal to N
// calls of warp_sum_canon: at every butterfly level each lane adds its
// partner's partial of the SAME value to its own (own + partner), exactly
// the pairs warp_sum_canon adds; the first log2(M) levels (M = N rounded up
// to a power of two) only split the values between the two lanes of a pair
// instead of computing both halves in both, so N values cost M - 1 + 5 -
// log2(M) shuffles and adds instead of 5 N.  On return, the total of value i
// is in the lanes with warp_multi_index<N>(lane) == i.
template <int N>
struct WarpMulti {
    static constexpr int M = N <= 1 ? 1 : N <= 2 ? 2 : N <= 4 ? 4 : N <= 8 ? 8 : N <= 16 ? 16 : 32;
};

template <int N>
__device__ __forceinline__ double warp_sum_multi(const double (&v)[N], int lane) {
    constexpr int M = WarpMulti<N>::M;
    double w[M];
#pragma unroll
    for (int i = 0; i < M; ++i) w[i] = i < N ? v[i] : 0.0;
    int o = 16;
#pragma unroll
    for (int h = M / 2; h >= 1; h >>= 1, o >>= 1) {
        const bool up = (lane & o) != 0;
#pragma unroll
        for (int i = 0; i < h; ++i) {
            const double send = up ? w[i] : w[i + h];
            const double keep = up ? w[i + h] : w[i];
            w[i] = __dadd_rn(keep, __shfl_xor_sync(0xffffffffu, send, o));
        }
    }
#pragma unroll
    for (; o > 0; o >>= 1) w[0] = __dadd_rn(w[0], __shfl_xor_sync(0xffffffffu, w[0], o));
    return w[0];
}

template <int N>
__device__ __forceinline__ int warp_multi_index(int lane) {
    constexpr int M = WarpMulti<N>::M;
    int idx = 0, o = 16;
#pragma unroll
    for (int h = M / 2; h >= 1; h >>= 1, o >>= 1)
        if (lane & o) idx += h;
    return idx;
}

// The N canonical warp sums of v (warp_sum_multi) stored by one lane each:
// dst[i * stride] = the warp total of value i.  Bitwise equal to N
// warp_sum_canon calls stored by lane 0.
template <int N>
__device__ __forceinline__ void warp_sums_store(const double (&v)[N], int lane, double *dst, int stride) {
    constexpr int M = WarpMulti<N>::M;
    const double s = warp_sum_multi<N>(v, lane);
    const int i = warp_multi_index<N>(lane);
    if (i < N && (lane & (32 / M - 1)) == 0) dst[i * stride] = s;
}

// Canonical block tree over n values v[0..n) (stride `stride`) computed by a
// block of RED_THREADS threads: thread t sums v[t], v[t+256], ... in order,
// then a fixed halving tree.  Must be called by all RED_THREADS threads;
// `sh` is RED_THREADS doubles of shared memory.  Returns the sum in all
// threads.
__device__ __forceinline__ double block_tree_sum(const double *v, int64_t n, double *sh) {
    const int t = threadIdx.x;
    double acc = 0.0;
    for (int64_t i = t; i < n; i += RED_THREADS) acc = __dadd_rn(acc, v[i]);
    sh[t] = acc;
    __syncthreads();
#pragma unroll
    for (int s = RED_THREADS / 2; s > 0; s >>= 1) {
        if (t < s) sh[t] = __dadd_rn(sh[t], sh[t + s]);
        __syncthreads();
    }
    double r = sh[0];
    __syncthreads();
    return r;
}

// Per-chunk tile-partial staging for z-march kernels with blockDim
// (DOT_TX, DOT_TY): warp w = threadIdx.y owns one x-row of the tile.
// After the chunk, tile value = ((w0 + w1) + w2) + ... + w7 per plane.
template <int ZC>
struct TileStage {
    double w[ZC][DOT_TY];
};

template <int ZC>
__device__ __forceinline__ void tile_stage_put(TileStage<ZC> &st, int zi, double v) {
    v = warp_sum_canon(v);
    if (threadIdx.x == 0) st.w[zi][threadIdx.y] = v;
}

// write the tile partials of planes [0, nplanes) of the chunk; plane index in
// the global tile-partial array = pbase + zi.  Call after __syncthreads().
template <int ZC>
__device__ __forceinline__ void tile_stage_flush(const TileStage<ZC> &st, int nplanes,
                                                 double *tp, int64_t pbase, int T, int tile) {
    int t = threadIdx.y * DOT_TX + threadIdx.x;
    if (t < nplanes) {
        double s = st.w[t][0];
#pragma unroll
        for (int w = 1; w < DOT_TY; ++w) s = __dadd_rn(s, st.w[t][w]);
        tp[(pbase + t) * (int64_t)T + tile] = s;
    }
}

// ---- counter-based fill (same generator as synth/, own implementation) -----
__device__ __forceinline__ uint64_t nb_mix64(uint64_t z) {
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ull;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBull;
    z ^= z >> 31;
    return z;
}

__device__ __forceinline__ double nb_gen(int kind, uint64_t seed, uint64_t gidx, double a, double b,
                                         int x, int y, int z, double h) {
    if (kind == NB_FILL_CONST) return a;
    if (kind == NB_FILL_POISSON_RHS) {
        // b = (h*h) * (((gy*gz + gx*gz) + gx*gy) * 2), g(t) = t*(1-t), t = (i+1)*h
        double tx = __dmul_rn((double)(x + 1), h), ty = __dmul_rn((double)(y + 1), h),
               tz = __dmul_rn((double)(z + 1), h);
        double gx = __dmul_rn(tx, __dsub_rn(1.0, tx)), gy = __dmul_rn(ty, __dsub_rn(1.0, ty)),
               gz = __dmul_rn(tz, __dsub_rn(1.0, tz));
        double f = __dadd_rn(__dadd_rn(__dmul_rn(gy, gz), __dmul_rn(gx, gz)), __dmul_rn(gx, gy));
        f = __dmul_rn(f, 2.0);
        return __dmul_rn(__dmul_rn(h, h), f);
    }
    uint64_t hsh = nb_mix64(seed * 0x9E3779B97F4A7C15ull + gidx + 1ull);
    if (kind == NB_FILL_UNIFORM) {
        double u = (double)(hsh >> 11) * 0x1p-53;
        return __dadd_rn(a, __dmul_rn(__dsub_rn(b, a), u));
    }
    // INT_UNIFORM: a + (h mod (b - a + 1))
    int64_t lo = (int64_t)a, hi = (int64_t)b;
    uint64_t span = (uint64_t)(hi - lo + 1);
    return (double)((int64_t)(hsh % span) + lo);
}

