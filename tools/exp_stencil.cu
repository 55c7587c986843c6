// Standalone micro-benchmark of CG phase-B-shaped kernels at 512^3 fp64
// (24 B/cell: read p, r; write r), to locate where stencil kernels lose
// bandwidth against a plain streaming kernel.  Not part of libnb.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o exp_stencil tools/exp_stencil.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int NX = 512, NY = 512, NZ = 512;
constexpr long PS = (long)NX * NY;

__device__ __forceinline__ double wsum(double v) {
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// V0: streaming, no stencil: r = r - a*p
__global__ void v0(const double *__restrict__ p, double *__restrict__ r, double a, long n) {
    for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < n; i += (long)gridDim.x * blockDim.x)
        r[PS + i] = fma(-a, p[PS + i], r[PS + i]);
}

// V1: flat 7-point, one cell per thread, CTA 32x8 of one plane, optional dot
template <bool DOT>
__global__ void v1(const double *__restrict__ p, double *__restrict__ r, double a, double *tp) {
    __shared__ double sw[8];
    const int x = blockIdx.x * 32 + threadIdx.x, y = blockIdx.y * 8 + threadIdx.y, z = blockIdx.z;
    const long i = (long)(z + 1) * PS + (long)y * NX + x;
    double c = p[i];
    double s = (x > 0 ? p[i - 1] : 0.0) + (x < NX - 1 ? p[i + 1] : 0.0);
    s += (y > 0 ? p[i - NX] : 0.0);
    s += (y < NY - 1 ? p[i + NX] : 0.0);
    s += p[i - PS];
    s += p[i + PS];
    double q = fma(6.0, c, -s);
    double rn = fma(-a, q, r[i]);
    r[i] = rn;
    if (DOT) {
        double v = wsum(rn * rn);
        if (threadIdx.x == 0) sw[threadIdx.y] = v;
        __syncthreads();
        if (threadIdx.x == 0 && threadIdx.y == 0) {
            double t = sw[0];
            for (int k = 1; k < 8; ++k) t += sw[k];
            tp[(long)z * 1024 + blockIdx.y * 16 + blockIdx.x] = t;
        }
    }
}

// V2: z-march, one cell per thread, ZC planes per CTA, L1 neighbours, optional dot
template <bool DOT, int ZC>
__global__ void v2(const double *__restrict__ p, double *__restrict__ r, double a, double *tp) {
    __shared__ double sw[ZC][8];
    const int x = blockIdx.x * 32 + threadIdx.x, y = blockIdx.y * 8 + threadIdx.y;
    const int zs = blockIdx.z * ZC;
    long i = (long)(zs + 1) * PS + (long)y * NX + x;
    double below = p[i - PS], c = p[i];
    for (int z = zs; z < zs + ZC; ++z, i += PS) {
        double above = p[i + PS];
        double s = (x > 0 ? p[i - 1] : 0.0) + (x < NX - 1 ? p[i + 1] : 0.0);
        s += (y > 0 ? p[i - NX] : 0.0);
        s += (y < NY - 1 ? p[i + NX] : 0.0);
        s += below;
        s += above;
        double q = fma(6.0, c, -s);
        double rn = fma(-a, q, r[i]);
        r[i] = rn;
        if (DOT) {
            double v = wsum(rn * rn);
            if (threadIdx.x == 0) sw[z - zs][threadIdx.y] = v;
        }
        below = c;
        c = above;
    }
    if (DOT) {
        __syncthreads();
        int t = threadIdx.y * 32 + threadIdx.x;
        if (t < ZC) {
            double s = sw[t][0];
            for (int k = 1; k < 8; ++k) s += sw[t][k];
            tp[(long)(zs + t) * 1024 + blockIdx.y * 16 + blockIdx.x] = s;
        }
    }
}


// V3: z-march, per-plane products staged in shared memory, butterflies of
// all ZC planes batched at the end of the chunk (independent chains)
template <int ZC>
__global__ void v3(const double *__restrict__ p, double *__restrict__ r, double a, double *tp) {
    __shared__ double sp[ZC][8][32];
    __shared__ double sw[ZC][8];
    const int x = blockIdx.x * 32 + threadIdx.x, y = blockIdx.y * 8 + threadIdx.y;
    const int zs = blockIdx.z * ZC;
    long i = (long)(zs + 1) * PS + (long)y * NX + x;
    double below = p[i - PS], c = p[i];
    for (int z = zs; z < zs + ZC; ++z, i += PS) {
        double above = p[i + PS];
        double s = (x > 0 ? p[i - 1] : 0.0) + (x < NX - 1 ? p[i + 1] : 0.0);
        s += (y > 0 ? p[i - NX] : 0.0);
        s += (y < NY - 1 ? p[i + NX] : 0.0);
        s += below;
        s += above;
        double q = fma(6.0, c, -s);
        double rn = fma(-a, q, r[i]);
        r[i] = rn;
        sp[z - zs][threadIdx.y][threadIdx.x] = rn * rn;
        below = c;
        c = above;
    }
    __syncwarp();
#pragma unroll
    for (int k = 0; k < ZC; ++k) {
        double v = wsum(sp[k][threadIdx.y][threadIdx.x]);
        if (threadIdx.x == 0) sw[k][threadIdx.y] = v;
    }
    __syncthreads();
    int t = threadIdx.y * 32 + threadIdx.x;
    if (t < ZC) {
        double s = sw[t][0];
        for (int k = 1; k < 8; ++k) s += sw[t][k];
        tp[(long)(zs + t) * 1024 + blockIdx.y * 16 + blockIdx.x] = s;
    }
}

// V4: v2 with the z loop unrolled by 2
template <int ZC>
__global__ void v4(const double *__restrict__ p, double *__restrict__ r, double a, double *tp) {
    __shared__ double sw[ZC][8];
    const int x = blockIdx.x * 32 + threadIdx.x, y = blockIdx.y * 8 + threadIdx.y;
    const int zs = blockIdx.z * ZC;
    long i = (long)(zs + 1) * PS + (long)y * NX + x;
    double below = p[i - PS], c = p[i];
#pragma unroll 2
    for (int z = zs; z < zs + ZC; ++z, i += PS) {
        double above = p[i + PS];
        double s = (x > 0 ? p[i - 1] : 0.0) + (x < NX - 1 ? p[i + 1] : 0.0);
        s += (y > 0 ? p[i - NX] : 0.0);
        s += (y < NY - 1 ? p[i + NX] : 0.0);
        s += below;
        s += above;
        double q = fma(6.0, c, -s);
        double rn = fma(-a, q, r[i]);
        r[i] = rn;
        double v = wsum(rn * rn);
        if (threadIdx.x == 0) sw[z - zs][threadIdx.y] = v;
        below = c;
        c = above;
    }
    __syncthreads();
    int t = threadIdx.y * 32 + threadIdx.x;
    if (t < ZC) {
        double s = sw[t][0];
        for (int k = 1; k < 8; ++k) s += sw[t][k];
        tp[(long)(zs + t) * 1024 + blockIdx.y * 16 + blockIdx.x] = s;
    }
}

template <typename F>
float timeit(F f, int reps = 20) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    f();
    cudaEventRecord(a);
    for (int k = 0; k < reps; ++k) f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    return ms / reps;
}

int main() {
    const long n = PS * NZ, tot = PS * (NZ + 2);
    double *p, *r, *tp;
    cudaMalloc(&p, tot * 8);
    cudaMalloc(&r, tot * 8);
    cudaMalloc(&tp, 1024L * 512 * 8);
    cudaMemset(p, 0, tot * 8);
    cudaMemset(r, 0, tot * 8);
    const double bytes = 24.0 * n;
    auto rep = [&](const char *nm, float ms) { printf("%-28s %8.3f ms  %7.2f TB/s\n", nm, ms, bytes / ms / 1e9); };
    rep("v0 stream", timeit([&] { v0<<<148 * 16, 256>>>(p, r, 1e-3, n); }));
    dim3 b(32, 8);
    rep("v1 flat nodot", timeit([&] { v1<false><<<dim3(16, 64, NZ), b>>>(p, r, 1e-3, tp); }));
    rep("v1 flat dot", timeit([&] { v1<true><<<dim3(16, 64, NZ), b>>>(p, r, 1e-3, tp); }));
    rep("v2 zmarch32 nodot", timeit([&] { v2<false, 32><<<dim3(16, 64, NZ / 32), b>>>(p, r, 1e-3, tp); }));
    rep("v2 zmarch32 dot", timeit([&] { v2<true, 32><<<dim3(16, 64, NZ / 32), b>>>(p, r, 1e-3, tp); }));
    rep("v2 zmarch8 dot", timeit([&] { v2<true, 8><<<dim3(16, 64, NZ / 8), b>>>(p, r, 1e-3, tp); }));
    rep("v2 zmarch4 dot", timeit([&] { v2<true, 4><<<dim3(16, 64, NZ / 4), b>>>(p, r, 1e-3, tp); }));
    rep("v3 staged8", timeit([&] { v3<8><<<dim3(16, 64, NZ / 8), b>>>(p, r, 1e-3, tp); }));
    rep("v3 staged16", timeit([&] { v3<16><<<dim3(16, 64, NZ / 16), b>>>(p, r, 1e-3, tp); }));
    rep("v4 unroll2 zc32", timeit([&] { v4<32><<<dim3(16, 64, NZ / 32), b>>>(p, r, 1e-3, tp); }));
    rep("v0 stream (again)", timeit([&] { v0<<<148 * 16, 256>>>(p, r, 1e-3, n); }));
    rep("v2 zmarch32 nodot (again)", timeit([&] { v2<false, 32><<<dim3(16, 64, NZ / 32), b>>>(p, r, 1e-3, tp); }));
    rep("v2 zmarch32 dot (again)", timeit([&] { v2<true, 32><<<dim3(16, 64, NZ / 32), b>>>(p, r, 1e-3, tp); }));
    cudaError_t e = cudaDeviceSynchronize();
    printf("status %s\n", cudaGetErrorString(e));
    return 0;
}
