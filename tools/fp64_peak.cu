// Measured FP64 FMA throughput of this B200 (the ALU roofline denominator of
// the FEM operator).  Each thread runs 8 independent DFMA
// chains; all SMs, several CTAs per SM; CUDA-event timed, best of 10.
// Not part of libnb.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_peak tools/fp64_peak.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int CH = 8;

__global__ void __launch_bounds__(256) k_dfma(double *out, double a, double b, int iters) {
    double v[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) v[c] = threadIdx.x * 1e-3 + c;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int k = 0; k < 16; ++k)
#pragma unroll
            for (int c = 0; c < CH; ++c) v[c] = fma(v[c], a, b);
    }
    double s = 0.0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += v[c];
    if (s == 12345.678) out[0] = s;  // keep the chains alive
}

int main() {
    int dev = 0, sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
    double *out;
    cudaMalloc(&out, 8);
    const int iters = 4096, threads = 256;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int per_sm : {4, 8}) {
        const int blocks = sms * per_sm;
        k_dfma<<<blocks, threads>>>(out, 0.999999, 1e-7, 64);
        float best = 1e30f;
        for (int rep = 0; rep < 10; ++rep) {
            cudaEventRecord(e0);
            k_dfma<<<blocks, threads>>>(out, 0.999999, 1e-7, iters);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        const double flop = 2.0 * CH * 16.0 * iters * (double)blocks * threads;
        const double tf = flop / (best * 1e-3) / 1e12;
        printf("{\"sms\": %d, \"clock_max_mhz\": %d, \"ctas_per_sm\": %d, \"ms\": %.4f, \"fp64_tflops\": %.3f, "
               "\"dfma_per_sm_per_clk_at_max\": %.2f}\n",
               sms, clk / 1000, per_sm, best, tf, tf * 1e12 / 2.0 / sms / (clk * 1e3));
    }
    return cudaGetLastError() != cudaSuccess;
}
