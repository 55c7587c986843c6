// Minimal TMA (cp.async.bulk.tensor.3d) check on fp64 boxes with negative
// coordinates (zero fill) — isolates descriptor / PTX issues from libnb.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_test tools/tma_test.cu
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                  const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

__global__ void k(const __grid_constant__ CUtensorMap m, double *out, int c0, int c1, int c2, int bxk) {
    __shared__ __align__(128) double buf[10][34];
    __shared__ __align__(8) uint64_t bar;
    uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar), d = (uint32_t)__cvta_generic_to_shared(&buf[0][0]);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(10 * bxk * 8) : "memory");
        asm volatile(
            "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::
                "r"(d),
            "l"(reinterpret_cast<uint64_t>(&m)), "r"(c0), "r"(c1), "r"(c2), "r"(b)
            : "memory");
    }
    uint32_t done = 0;
    while (!done)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(done)
                     : "r"(b)
                     : "memory");
    for (int i = threadIdx.x; i < 340; i += blockDim.x) out[i] = (&buf[0][0])[i];
}

int main(int argc, char **argv) {
    int c0 = argc > 1 ? atoi(argv[1]) : -1, c1 = argc > 2 ? atoi(argv[2]) : 55;
    int bx = argc > 3 ? atoi(argv[3]) : 34;
    const int nx = 64, ny = 64, nz = 66;
    std::vector<double> h((size_t)nx * ny * nz);
    for (size_t i = 0; i < h.size(); ++i) h[i] = (double)i;
    double *d, *o;
    cudaMalloc(&d, h.size() * 8);
    cudaMalloc(&o, 340 * 8);
    cudaMemcpy(d, h.data(), h.size() * 8, cudaMemcpyHostToDevice);
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
    EncodeTiledFn fn = (EncodeTiledFn)p;
    CUtensorMap m;
    cuuint64_t dims[3] = {nx, ny, nz}, strides[2] = {nx * 8, (cuuint64_t)nx * ny * 8};
    cuuint32_t box[3] = {(cuuint32_t)bx, 10, 1}, es[3] = {1, 1, 1};
    CUresult r = fn(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, d, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode %d\n", (int)r);
    k<<<1, 128>>>(m, o, c0, c1, 0, bx);
    cudaError_t e = cudaDeviceSynchronize();
    printf("kernel %s\n", cudaGetErrorString(e));
    std::vector<double> ho(340);
    cudaMemcpy(ho.data(), o, 340 * 8, cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int yy = 0; yy < 10; ++yy)
        for (int xx = 0; xx < 34; ++xx) {
            int x = xx + c0, y = c1 + yy;
            double exp = (x >= 0 && x < nx && y < ny && y >= 0 && xx < bx) ? (double)(x + nx * y) : 0.0;
            if (xx < bx && ho[yy * bx + xx] != exp) ++bad;
        }
    printf("mismatches %d\n", bad);
    return 0;
}
