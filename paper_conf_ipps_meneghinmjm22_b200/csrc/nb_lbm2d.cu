// nb_lbm2d.cu — D2Q9 BGK, the 2-D Kármán vortex street of PAPER.md Table I
// (L398-L439).  The paper names the application only;
// lattice and boundaries are the readings of DESIGN.md §3 (the oracle
// or_d2q9_step follows them step by step):
//   D2Q9, pull stream + BGK collide fused (as the 3-D kernel), fp32;
//   solid cylinder (x-cx)^2 + (y-cy)^2 <= r^2: half-way bounce-back, solid
//   cells hold 0; channel: y periodic, inflow equilibrium (rho 1, u_in) for
//   sources left of x = 0, zero-gradient outflow (sources clamped to column
//   nx-1); or a fully periodic box.
// The field lives on a grid of Nz = 1 (one plane), 9 fp32 components, SoA.
#include <cstring>

#include "nb_internal.cuh"

nb_status nb_launch_check(const char *what);

namespace {
__device__ __host__ constexpr int CX9(int i) {
    constexpr int t[9] = {0, 1, -1, 0, 0, 1, -1, 1, -1};
    return t[i];
}
__device__ __host__ constexpr int CY9(int i) {
    constexpr int t[9] = {0, 0, 0, 1, -1, 1, -1, -1, 1};
    return t[i];
}
__device__ __host__ constexpr int OPP9(int i) {
    constexpr int t[9] = {0, 2, 1, 4, 3, 6, 5, 8, 7};
    return t[i];
}
__device__ __host__ constexpr float W9(int i) { return i == 0 ? 4.0f / 9.0f : (i < 5 ? 1.0f / 9.0f : 1.0f / 36.0f); }

__device__ __forceinline__ float feq9(int i, float rho, float ux, float uy) {
    const float cu = (float)CX9(i) * ux + (float)CY9(i) * uy;
    return W9(i) * rho * (1.0f + 3.0f * cu + 4.5f * cu * cu - 1.5f * (ux * ux + uy * uy));
}

__device__ __forceinline__ bool solid9(int x, int y, const nb_d2q9_params &p) {
    const long long dx = x - p.cx, dy = y - p.cy;
    return p.r >= 0 && dx * dx + dy * dy <= (long long)p.r * p.r;
}
}  // namespace

struct D2q9Args {
    const float *fin;
    float *fout;
    int64_t cs;  // component stride (elements)
    int nx, ny;
    int64_t pitch, plane;  // row pitch; offset of plane 0 (= ps)
    nb_d2q9_params p;
    float omega, u_in;
};

__global__ void __launch_bounds__(128) k_lbm_d2q9(D2q9Args A) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y;
    if (x >= A.nx) return;
    const int64_t cell = A.plane + (int64_t)y * A.pitch + x;
    if (solid9(x, y, A.p)) {
#pragma unroll
        for (int i = 0; i < 9; ++i) A.fout[i * A.cs + cell] = 0.0f;
        return;
    }
    float f[9];
    const bool interior = x > 0 && x < A.nx - 1 && y > 0 && y < A.ny - 1 &&
                          (A.p.r < 0 || (x - A.p.cx) * (long long)(x - A.p.cx) + (y - A.p.cy) * (long long)(y - A.p.cy) >
                                            (long long)(A.p.r + 2) * (A.p.r + 2));
    if (interior) {  // no boundary and no solid within reach: 9 uniform-offset loads
#pragma unroll
        for (int i = 0; i < 9; ++i) f[i] = __ldg(A.fin + i * A.cs + cell - (int64_t)CY9(i) * A.pitch - CX9(i));
    } else {
#pragma unroll
        for (int i = 0; i < 9; ++i) {
            int sx = x - CX9(i), sy = y - CY9(i);
            sy = sy < 0 ? sy + A.ny : (sy >= A.ny ? sy - A.ny : sy);
            if (A.p.bc == 1) sx = sx < 0 ? sx + A.nx : (sx >= A.nx ? sx - A.nx : sx);
            if (sx < 0) {
                f[i] = feq9(i, 1.0f, A.u_in, 0.0f);
                continue;
            }
            if (sx >= A.nx) sx = A.nx - 1;
            f[i] = solid9(sx, sy, A.p) ? __ldg(A.fin + OPP9(i) * A.cs + cell)
                                       : __ldg(A.fin + i * A.cs + A.plane + (int64_t)sy * A.pitch + sx);
        }
    }
    float rho = 0.f, jx = 0.f, jy = 0.f;
#pragma unroll
    for (int i = 0; i < 9; ++i) {
        rho += f[i];
        jx += (float)CX9(i) * f[i];
        jy += (float)CY9(i) * f[i];
    }
    const float ux = jx / rho, uy = jy / rho;
#pragma unroll
    for (int i = 0; i < 9; ++i) __stcs(A.fout + i * A.cs + cell, f[i] - A.omega * (f[i] - feq9(i, rho, ux, uy)));
}

__global__ void k_d2q9_init(float *f, int64_t cs, int64_t n, float rho, float ux, float uy) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
#pragma unroll
        for (int i = 0; i < 9; ++i) f[i * cs + e] = feq9(i, rho, ux, uy);
}

static nb_status d2q9_check(const nb_field *f) {
    if (!f) NB_FAIL(NB_EINVAL, "NULL field");
    const nb_grid *g = f->g;
    if (f->dt != NB_F32 || f->card != 9) NB_FAIL(NB_EMISMATCH, "D2Q9 needs an fp32 field of cardinality 9");
    NB_LAYOUTS(f, 1 << NB_SOA, "D2Q9");
    if (g->sparse || g->nz != 1 || g->nparts != 1)
        NB_FAIL(NB_EUNSUPPORTED, "D2Q9: a dense grid of one plane (Nz = 1) on one partition");
    return NB_OK;
}

extern "C" nb_status nb_d2q9_init(nb_field *f, double rho0, double ux, double uy) {
    NB_TRY(d2q9_check(f));
    nb_grid *g = f->g;
    cudaSetDevice(g->device);
    const int64_t cs = f->ps * 3;
    LaunchScope ls(g, g->cs, "k_d2q9_init");
    k_d2q9_init<<<296, 256, 0, g->cs>>>((float *)f->base[0], cs, cs, (float)rho0, (float)ux, (float)uy);
    return nb_launch_check("k_d2q9_init");
}

extern "C" nb_status nb_d2q9_step(nb_field **pfin, nb_field **pfout, const nb_d2q9_params *prm, int32_t nsteps) {
    if (!pfin || !pfout || !prm) NB_FAIL(NB_EINVAL, "nb_d2q9_step: NULL argument");
    nb_field *fin = *pfin, *fout = *pfout;
    NB_TRY(d2q9_check(fin));
    NB_TRY(d2q9_check(fout));
    if (fin == fout || fin->g != fout->g) NB_FAIL(NB_EINVAL, "two distinct fields of one grid");
    if (prm->bc != 0 && prm->bc != 1) NB_FAIL(NB_EINVAL, "bc: 0 channel, 1 periodic");
    if (nsteps < 0) NB_FAIL(NB_EINVAL, "nsteps < 0");
    nb_grid *g = fin->g;
    cudaSetDevice(g->device);
    D2q9Args A;
    memset(&A, 0, sizeof(A));
    A.cs = fin->ps * 3;
    A.nx = g->nx;
    A.ny = g->ny;
    A.pitch = fin->pitch;
    A.plane = fin->ps;
    A.p = *prm;
    A.omega = (float)prm->omega;
    A.u_in = (float)prm->u_in;
    dim3 blk(128), grd((g->nx + 127) / 128, g->ny);
    for (int t = 0; t < nsteps; ++t) {
        A.fin = (const float *)fin->base[0];
        A.fout = (float *)fout->base[0];
        LaunchScope ls(g, g->cs, "k_lbm_d2q9");
        k_lbm_d2q9<<<grd, blk, 0, g->cs>>>(A);
        NB_TRY(nb_launch_check("k_lbm_d2q9"));
        std::swap(fin, fout);
    }
    *pfin = fin;
    *pfout = fout;
    return NB_OK;
}
