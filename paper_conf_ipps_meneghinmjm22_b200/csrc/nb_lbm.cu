// nb_lbm.cu — D3Q19 BGK lattice Boltzmann, twoPop pull scheme, fused
// collide-and-stream (§VI-A: "Collide and streaming steps
// are fused into a single kernel", twoPop "works on two buffers ... swapped").
//
// Per cell (the formulas are the SURVEY.md §8(c) c6 reading):
//   f_i = fin_i(x - c_i)                 (pull: own-compute rule, L246)
//       | fin_opp(i)(x) + 6 w_i rho_w (c_i . u_lid)[lid]   (half-way bounce-back)
//   rho = sum f_i ; u = sum c_i f_i / rho
//   feq_i = w_i rho (1 + 3 c.u + 4.5 (c.u)^2 - 1.5 |u|^2)
//   fout_i(x) = f_i - omega (f_i - feq_i)
// fp32 storage and arithmetic, SoA [c][zl][y][x].  Algorithmic traffic
// 19 loads + 19 stores of 4 B = 152 B per cell per step.
//
// Velocity order (halo-contiguous): 0 rest; 1-4 (+-x, +-y); 5-8 xy diagonals;
// 9-13 c_z = +1; 14-18 c_z = -1.
#include <algorithm>
#include <cstring>

#include "nb_device.cuh"
#include "nb_internal.cuh"

namespace {
__device__ __host__ constexpr int CXv(int i) {
    constexpr int t[19] = {0, 1, -1, 0, 0, 1, -1, 1, -1, 0, 1, -1, 0, 0, 0, -1, 1, 0, 0};
    return t[i];
}
__device__ __host__ constexpr int CYv(int i) {
    constexpr int t[19] = {0, 0, 0, 1, -1, 1, -1, -1, 1, 0, 0, 0, 1, -1, 0, 0, 0, -1, 1};
    return t[i];
}
__device__ __host__ constexpr int CZv(int i) {
    constexpr int t[19] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 1, 1, 1, 1, 1, -1, -1, -1, -1, -1};
    return t[i];
}
__device__ __host__ constexpr int OPPv(int i) {
    constexpr int t[19] = {0, 2, 1, 4, 3, 6, 5, 8, 7, 14, 15, 16, 17, 18, 9, 10, 11, 12, 13};
    return t[i];
}
__device__ __host__ constexpr float Wv(int i) {
    return i == 0 ? 1.0f / 3.0f : (CXv(i) * CXv(i) + CYv(i) * CYv(i) + CZv(i) * CZv(i) == 1 ? 1.0f / 18.0f : 1.0f / 36.0f);
}
}  // namespace

struct LbmArgs {
    const float *fin[Q19];   // component base pointers (plane zl = -1, row 0)
    float *fout[Q19];
    float *rem_lo[Q19];      // lower neighbour's fout components at its high halo plane (14..18 used)
    float *rem_hi[Q19];      // upper neighbour's fout components at its low halo plane (9..13 used)
    PGeo g;
    float omega, ulid, rho_w;
};

// BGK collision of the gathered populations and the streaming store (shared
// by the interior fast path and the boundary path: same code, same bits)
__device__ __forceinline__ void lbm_collide(const float (&f)[Q19], float om, float (&o)[Q19]) {
    float rho = 0.f, jx = 0.f, jy = 0.f, jz = 0.f;
#pragma unroll
    for (int i = 0; i < Q19; ++i) {
        rho += f[i];
        if (CXv(i) == 1) jx += f[i];
        if (CXv(i) == -1) jx -= f[i];
        if (CYv(i) == 1) jy += f[i];
        if (CYv(i) == -1) jy -= f[i];
        if (CZv(i) == 1) jz += f[i];
        if (CZv(i) == -1) jz -= f[i];
    }
    // one reciprocal instead of three divisions; feq = (w rho) (base + cu (3 + 4.5 cu))
    // with base = 1 - 1.5 |u|^2 and w rho per weight class
    const float ir = 1.0f / rho;
    const float ux = jx * ir, uy = jy * ir, uz = jz * ir;
    const float usq = ux * ux + uy * uy + uz * uz;
    const float base = 1.0f - 1.5f * usq;
    const float r0 = (1.0f / 3.0f) * rho, r1 = (1.0f / 18.0f) * rho, r2 = (1.0f / 36.0f) * rho;
#pragma unroll
    for (int i = 0; i < Q19; ++i) {
        const float cu = (float)CXv(i) * ux + (float)CYv(i) * uy + (float)CZv(i) * uz;
        const float wr = i == 0 ? r0 : (CXv(i) * CXv(i) + CYv(i) * CYv(i) + CZv(i) * CZv(i) == 1 ? r1 : r2);
        const float feq = wr * fmaf(cu, fmaf(4.5f, cu, 3.0f), base);
        o[i] = fmaf(-om, f[i] - feq, f[i]);
    }
}

// ES: element stride of a cell index (1: SOA / SOA_PLANE, 19: AOS)
template <int ES>
__device__ __forceinline__ void lbm_collide_store(const float (&f)[Q19], const LbmArgs &A, int64_t cell,
                                                  int zl, int64_t row) {
    float o[Q19];
    lbm_collide(f, A.omega, o);
#pragma unroll
    for (int i = 0; i < Q19; ++i) __stcs(A.fout[i] + cell * ES, o[i]);
    // halo transfer fused into the producing kernel: outgoing populations of
    // the boundary planes go straight into the neighbours' halo planes
    if (zl == 0 && A.rem_lo[14]) {
#pragma unroll
        for (int i = 14; i < 19; ++i) A.rem_lo[i][row * ES] = o[i];
    }
    if (zl == A.g.nzl - 1 && A.rem_hi[9]) {
#pragma unroll
        for (int i = 9; i < 14; ++i) A.rem_hi[i][row * ES] = o[i];
    }
}

template <bool PERIODIC, int ES>
// x-threads per CTA of the twoPop D3Q19 step (256: 3.18 -> 3.10 ms at
// 512^3 against 128; 512 is slower, 3.75)
#ifndef NB_LBM_BX
#define NB_LBM_BX 256
#endif
__global__ void __launch_bounds__(NB_LBM_BX) k_lbm_d3q19(LbmArgs A, int zb) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x;
    const int y = blockIdx.y;
    const int zl = zb + blockIdx.z;
    const PGeo &g = A.g;
    if (x >= g.nx) return;
    const int gz = g.z0 + zl;
    const int64_t row = (int64_t)y * g.pitch + x;
    const int64_t cell = (int64_t)(zl + 1) * g.ps + row;
    float f[Q19];
    const bool interior = x > 0 && x < g.nx - 1 && y > 0 && y < g.ny - 1 &&
                          (PERIODIC || (gz > 0 && gz < g.NZ - 1));
    if (interior) {
        // every source is in the slab or its halo planes: 19 independent
        // loads at uniform offsets
#pragma unroll
        for (int i = 0; i < Q19; ++i)
            f[i] = __ldg(A.fin[i] + (cell - (int64_t)CZv(i) * g.ps - (int64_t)CYv(i) * g.pitch - CXv(i)) * ES);
    } else {
#pragma unroll
        for (int i = 0; i < Q19; ++i) {
            int sx = x - CXv(i), sy = y - CYv(i), szl = zl - CZv(i);
            if (PERIODIC) {
                sx = sx < 0 ? sx + g.nx : (sx >= g.nx ? sx - g.nx : sx);
                sy = sy < 0 ? sy + g.ny : (sy >= g.ny ? sy - g.ny : sy);
                f[i] = __ldg(A.fin[i] + ((int64_t)(szl + 1) * g.ps + (int64_t)sy * g.pitch + sx) * ES);
            } else {
                // in-domain neighbour, or half-way bounce-back from the
                // opposite population of this cell (+ moving-lid term)
                const int sgz = gz - CZv(i);
                const bool inside = sx >= 0 && sx < g.nx && sy >= 0 && sy < g.ny && sgz >= 0 && sgz < g.NZ;
                const float *src = inside ? A.fin[i] + ((int64_t)(szl + 1) * g.ps + (int64_t)sy * g.pitch + sx) * ES
                                          : A.fin[OPPv(i)] + cell * ES;
                float v = __ldg(src);
                if (CXv(i) != 0 && sy == g.ny && sx >= 0 && sx < g.nx && sgz >= 0 && sgz < g.NZ)
                    v = v + 6.0f * Wv(i) * A.rho_w * ((float)CXv(i) * A.ulid);
                f[i] = v;
            }
        }
    }
    lbm_collide_store<ES>(f, A, cell, zl, row);
}

__global__ void __launch_bounds__(128) k_lbm_init(float *f, PGeo g, int64_t cs, int64_t es, float rho, float ux,
                                                  float uy, float uz) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y, zl = (int)blockIdx.z - 1;
    if (x >= g.nx) return;
    const int64_t cell = (int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x;
    const float usq = ux * ux + uy * uy + uz * uz;
#pragma unroll
    for (int i = 0; i < Q19; ++i) {
        float cu = (float)CXv(i) * ux + (float)CYv(i) * uy + (float)CZv(i) * uz;
        f[(int64_t)i * cs + cell * es] = Wv(i) * rho * (1.0f + 3.0f * cu + 4.5f * cu * cu - 1.5f * usq);
    }
}

// per-field addressing of the macroscopic kernel (the three fields may use
// different layouts): element (c, zl, y, x) at c*cs + ((zl+1)*ps + y*pitch + x)*es
struct LbmFa {
    int64_t ps, cs, es;
    __device__ __forceinline__ int64_t at(int c, int zl, int64_t row) const { return c * cs + ((zl + 1) * ps + row) * es; }
};
__global__ void __launch_bounds__(128) k_lbm_macro(const float *f, float *rho_o, float *u_o, PGeo g, LbmFa af,
                                                   LbmFa ar, LbmFa au) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y, zl = blockIdx.z;
    if (x >= g.nx) return;
    const int64_t row = (int64_t)y * g.pitch + x;
    float rho = 0.f, jx = 0.f, jy = 0.f, jz = 0.f;
#pragma unroll
    for (int i = 0; i < Q19; ++i) {
        float v = f[af.at(i, zl, row)];
        rho += v;
        jx += (float)CXv(i) * v;
        jy += (float)CYv(i) * v;
        jz += (float)CZv(i) * v;
    }
    rho_o[ar.at(0, zl, row)] = rho;
    u_o[au.at(0, zl, row)] = jx / rho;
    u_o[au.at(1, zl, row)] = jy / rho;
    u_o[au.at(2, zl, row)] = jz / rho;
}

static inline int64_t lcs(const nb_field *f, int p) { return nb_cstride(f, p); }

static nb_status lbm_check(const nb_field *f) {
    if (!f) NB_FAIL(NB_EINVAL, "NULL field");
    if (f->dt != NB_F32 || f->card != Q19) NB_FAIL(NB_EMISMATCH, "LBM needs an fp32 field of cardinality 19");
    return NB_OK;
}

// ===========================================================================
// D3Q19 on element-sparse domains ("the
// domain is free-form", L248 element-sparse grid).  Same pull step, with the
// sources looked up in an 18-direction connectivity table of the compact
// (z, y, x) cell order: -1 = no fluid source (inactive cell or outside the
// box: half-way bounce-back), -2 = beyond the moving lid (y = Ny face).
// One thread per active cell; the collision is the dense kernel's (bitwise:
// a full mask reproduces the dense grid).  Halos: the 5 populations with
// c_z = +1 up, the 5 with c_z = -1 down, contiguous segments.
// ===========================================================================
nb_status nb_sparse_slab_map(nb_grid *g, int p, uint8_t **d_mask, int32_t **d_map, int *slab_z0, int *nslab);
nb_status nb_sparse_halo_comps(nb_field *f, int c0u, int c1u, int c0d, int c1d);

__global__ void k_sp_conn19(const uint8_t *__restrict__ mask, const int32_t *__restrict__ map, int nx, int ny,
                            int slab_z0, int nslab, int z0, int NZ, int64_t hl, int64_t n, int32_t *conn19) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y, z = z0 + blockIdx.z;
    if (x >= nx) return;
    const int64_t plane = (int64_t)nx * ny;
    const int64_t cell = (int64_t)(z - slab_z0) * plane + (int64_t)y * nx + x;
    if (!mask[cell]) return;
    const int64_t j = (int64_t)map[cell] - hl;
#pragma unroll
    for (int q = 1; q < Q19; ++q) {
        const int sx = x - CXv(q), sy = y - CYv(q), sz = z - CZv(q);
        int32_t v = -1;
        if (sx >= 0 && sx < nx && sy >= 0 && sy < ny && sz >= 0 && sz < NZ && sz - slab_z0 >= 0 &&
            sz - slab_z0 < nslab) {
            const int64_t sc = (int64_t)(sz - slab_z0) * plane + (int64_t)sy * nx + sx;
            if (mask[sc]) v = map[sc];
        } else if (sy == ny && sx >= 0 && sx < nx && sz >= 0 && sz < NZ) {
            v = -2;
        }
        conn19[(int64_t)(q - 1) * n + j] = v;
    }
}

#ifndef NB_SPLBM_BX
#define NB_SPLBM_BX 32  // 1.41 -> 1.35 ms per step on the C4 sphere against 128 (64: 1.41)
#endif
__global__ void __launch_bounds__(NB_SPLBM_BX) k_sp_lbm(const float *__restrict__ fin, float *__restrict__ fout, int64_t cs,
                                                int64_t hl, int64_t n, const int32_t *__restrict__ conn19, float om,
                                                float ulid, float rho_w) {
    const int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (j >= n) return;
    const int64_t own = hl + j;
    int32_t src[Q19];
#pragma unroll
    for (int q = 1; q < Q19; ++q) src[q] = __ldg(conn19 + (int64_t)(q - 1) * n + j);
    float f[Q19];
    f[0] = __ldg(fin + own);
#pragma unroll
    for (int q = 1; q < Q19; ++q) {
        const int32_t k = src[q];
        float v = __ldg(k >= 0 ? fin + (int64_t)q * cs + k : fin + (int64_t)OPPv(q) * cs + own);
        if (CXv(q) != 0 && k == -2) v = v + 6.0f * Wv(q) * rho_w * ((float)CXv(q) * ulid);
        f[q] = v;
    }
    float o[Q19];
    lbm_collide(f, om, o);
#pragma unroll
    for (int q = 0; q < Q19; ++q) __stcs(fout + (int64_t)q * cs + own, o[q]);
}

__global__ void k_sp_lbm_init(float *f, int64_t cs, float rho, float ux, float uy, float uz) {
    const float usq = ux * ux + uy * uy + uz * uz;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < cs; e += (int64_t)gridDim.x * blockDim.x) {
#pragma unroll
        for (int i = 0; i < Q19; ++i) {
            float cu = (float)CXv(i) * ux + (float)CYv(i) * uy + (float)CZv(i) * uz;
            f[(int64_t)i * cs + e] = Wv(i) * rho * (1.0f + 3.0f * cu + 4.5f * cu * cu - 1.5f * usq);
        }
    }
}

__global__ void k_sp_lbm_macro(const float *f, float *rho_o, float *u_o, int64_t cs, int64_t cs_rho, int64_t cs_u,
                               int64_t hl, int64_t n) {
    const int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (j >= n) return;
    const int64_t e = hl + j;
    float rho = 0.f, jx = 0.f, jy = 0.f, jz = 0.f;
#pragma unroll
    for (int i = 0; i < Q19; ++i) {
        float v = f[(int64_t)i * cs + e];
        rho += v;
        jx += (float)CXv(i) * v;
        jy += (float)CYv(i) * v;
        jz += (float)CZv(i) * v;
    }
    (void)cs_rho;
    rho_o[e] = rho;
    u_o[e] = jx / rho;
    u_o[cs_u + e] = jy / rho;
    u_o[2 * cs_u + e] = jz / rho;
}

static nb_status sp_lbm_tables(nb_grid *g) {
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        NbSparsePart &sp = g->sp[p];
        if (sp.conn19) continue;
        uint8_t *d_mask = nullptr;
        int32_t *d_map = nullptr;
        int slab_z0 = 0, nslab = 0;
        nb_status s = nb_sparse_slab_map(g, p, &d_mask, &d_map, &slab_z0, &nslab);
        if (s == NB_OK && cudaMalloc(&sp.conn19, sizeof(int32_t) * 18 * std::max<int64_t>(sp.n, 1)) != cudaSuccess) {
            cudaGetLastError();
            nb_set_error("sparse LBM: cudaMalloc of the D3Q19 connectivity failed");
            s = NB_ENOMEM;
        }
        if (s == NB_OK && g->parts[p].nz() > 0) {
            dim3 blk(128), grd((g->nx + 127) / 128, g->ny, g->parts[p].nz());
            LaunchScope ls(g, g->cs, "k_sp_conn19");
            k_sp_conn19<<<grd, blk, 0, g->cs>>>(d_mask, d_map, g->nx, g->ny, slab_z0, nslab, g->parts[p].z0, g->nz,
                                                 sp.hl, sp.n, sp.conn19);
            s = nb_launch_check("k_sp_conn19");
            cudaStreamSynchronize(g->cs);
        }
        cudaFree(d_mask);
        cudaFree(d_map);
        if (s != NB_OK) return s;
    }
    return NB_OK;
}

static nb_status sp_lbm_step(nb_field **pfin, nb_field **pfout, const nb_lbm_params *prm, int nsteps) {
    nb_field *fin = *pfin, *fout = *pfout;
    nb_grid *g = fin->g;
    if (prm->bc != NB_LBM_CAVITY)
        NB_FAIL(NB_EUNSUPPORTED, "LBM on element-sparse grids: bounce-back (cavity) boundaries only");
    NB_TRY(sp_lbm_tables(g));
    NB_TRY(nb_sparse_halo_comps(fin, 9, 14, 14, 19));
    for (int t = 0; t < nsteps; ++t) {
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            const NbSparsePart &sp = g->sp[p];
            if (sp.n == 0) continue;
            LaunchScope ls(g, g->cs, "k_sp_lbm");
            k_sp_lbm<<<(unsigned)((sp.n + NB_SPLBM_BX - 1) / NB_SPLBM_BX), NB_SPLBM_BX, 0, g->cs>>>(
                (const float *)fin->base[p], (float *)fout->base[p], fin->pcs[p], sp.hl, sp.n, sp.conn19,
                (float)prm->omega, (float)prm->u_lid, (float)prm->rho_w);
            NB_TRY(nb_launch_check("k_sp_lbm"));
        }
        NB_TRY(nb_sparse_halo_comps(fout, 9, 14, 14, 19));
        std::swap(fin, fout);
    }
    *pfin = fin;
    *pfout = fout;
    return NB_OK;
}

extern "C" nb_status nb_lbm_init(nb_field *f, double rho0, const double u0[3]) {
    NB_TRY(lbm_check(f));
    if (!u0) NB_FAIL(NB_EINVAL, "u0 is NULL");
    nb_grid *g = f->g;
    cudaSetDevice(g->device);
    if (g->sparse) {
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            LaunchScope ls(g, g->cs, "k_lbm_init");
            k_sp_lbm_init<<<296, 256, 0, g->cs>>>((float *)f->base[p], f->pcs[p], (float)rho0, (float)u0[0],
                                                  (float)u0[1], (float)u0[2]);
            NB_TRY(nb_launch_check("k_sp_lbm_init"));
        }
        return NB_OK;
    }
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        PGeo geo = pgeo(f, p);
        dim3 blk(128), grd((g->nx + 127) / 128, g->ny, geo.nzl + 2);  // halo planes too
        LaunchScope ls(g, g->cs, "k_lbm_init");
        k_lbm_init<<<grd, blk, 0, g->cs>>>((float *)f->base[p], geo, lcs(f, p), f->es, (float)rho0, (float)u0[0],
                                           (float)u0[1], (float)u0[2]);
        NB_TRY(nb_launch_check("k_lbm_init"));
    }
    return NB_OK;
}

// neighbours for the LBM (ring when periodic)
static int lbm_lo(const nb_grid *g, int p, bool per) {
    if (g->parts[p].lo >= 0) return g->parts[p].lo;
    return per ? g->nparts - 1 : -1;
}
static int lbm_hi(const nb_grid *g, int p, bool per) {
    if (g->parts[p].hi >= 0) return g->parts[p].hi;
    return per ? 0 : -1;
}

// Halo of the 10 populations that cross z faces: my last plane's c_z=+1
// populations (9..13) -> upper neighbour's low halo; my first plane's c_z=-1
// populations (14..18) -> lower neighbour's high halo (ring when periodic).
// Local partners: device copies; remote partners: grouped NCCL send/recv in
// the canonical order of nb_halo_plan.
static nb_status lbm_halo(nb_field *f, bool per, cudaStream_t s) { return nb_halo_run(f, per, 9, 14, 14, 19, s); }

static nb_status launch_lbm(nb_grid *g, int p, nb_field *fin, nb_field *fout, const nb_lbm_params *prm, int zb,
                            int ze, bool remote_stores) {
    if (ze <= zb) return NB_OK;
    bool per = prm->bc == NB_LBM_PERIODIC;
    LbmArgs A;
    memset(&A, 0, sizeof(A));
    for (int i = 0; i < Q19; ++i) {
        A.fin[i] = (const float *)fin->base[p] + (int64_t)i * lcs(fin, p);
        A.fout[i] = (float *)fout->base[p] + (int64_t)i * lcs(fout, p);
    }
    A.g = pgeo(fin, p);
    A.omega = (float)prm->omega;
    A.ulid = (float)prm->u_lid;
    A.rho_w = (float)prm->rho_w;
    if (remote_stores) {
        int lo = lbm_lo(g, p, per), hi = lbm_hi(g, p, per);
        if (zb == 0 && nb_reachable(fout, lo))
            for (int i = 14; i < 19; ++i)
                A.rem_lo[i] = (float *)fout->base[lo] + (int64_t)i * lcs(fout, lo) +
                              (int64_t)(g->parts[lo].nz() + 1) * fout->ps * fout->es;
        if (ze == g->parts[p].nz() && nb_reachable(fout, hi))
            for (int i = 9; i < 14; ++i) A.rem_hi[i] = (float *)fout->base[hi] + (int64_t)i * lcs(fout, hi);
    }
    dim3 blk(NB_LBM_BX), grd((g->nx + NB_LBM_BX - 1) / NB_LBM_BX, g->ny, ze - zb);
    LaunchScope ls(g, g->cs, "k_lbm_d3q19");
    const bool aos = fin->layout == NB_AOS;
    if (per && aos)
        k_lbm_d3q19<true, Q19><<<grd, blk, 0, g->cs>>>(A, zb);
    else if (per)
        k_lbm_d3q19<true, 1><<<grd, blk, 0, g->cs>>>(A, zb);
    else if (aos)
        k_lbm_d3q19<false, Q19><<<grd, blk, 0, g->cs>>>(A, zb);
    else
        k_lbm_d3q19<false, 1><<<grd, blk, 0, g->cs>>>(A, zb);
    return nb_launch_check("k_lbm_d3q19");
}

// one step of fin into fout on the planes of view v of every local
// partition, halos as they are (the Skeleton's LBM container: its halo node
// runs before, explicitly); cavity boundaries
nb_status nb_lbm_view(nb_field *fin, nb_field *fout, const nb_lbm_params *prm, nb_view v) {
    NB_TRY(lbm_check(fin));
    NB_TRY(lbm_check(fout));
    if (fin->g != fout->g) NB_FAIL(NB_EMISMATCH, "fin and fout belong to different grids");
    if (fin->layout != fout->layout) NB_FAIL(NB_EMISMATCH, "fin and fout have different layouts");
    if (fin == fout) NB_FAIL(NB_EINVAL, "twoPop needs two distinct buffers");
    if (prm->bc != NB_LBM_CAVITY) NB_FAIL(NB_EUNSUPPORTED, "Skeleton LBM containers: cavity boundaries");
    nb_grid *g = fin->g;
    if (g->sparse) NB_FAIL(NB_EUNSUPPORTED, "Skeleton LBM containers: dense grids");
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p)
        for (auto rg : view_ranges(g, p, v)) NB_TRY(launch_lbm(g, p, fin, fout, prm, rg.first, rg.second, false));
    return NB_OK;
}

extern "C" nb_status nb_lbm_step(nb_field **pfin, nb_field **pfout, const nb_lbm_params *prm, int32_t nsteps,
                                 nb_occ occ) {
    NB_RANGE("nb_lbm_step");
    if (!pfin || !pfout || !prm) NB_FAIL(NB_EINVAL, "nb_lbm_step: NULL argument");
    nb_field *fin = *pfin, *fout = *pfout;
    NB_TRY(lbm_check(fin));
    NB_TRY(lbm_check(fout));
    if (fin->g != fout->g) NB_FAIL(NB_EMISMATCH, "fin and fout belong to different grids");
    if (fin->layout != fout->layout) NB_FAIL(NB_EMISMATCH, "fin and fout have different layouts");
    if (fin == fout) NB_FAIL(NB_EINVAL, "twoPop needs two distinct buffers");
    if (nsteps < 0) NB_FAIL(NB_EINVAL, "nsteps < 0");
    if (prm->bc != NB_LBM_CAVITY && prm->bc != NB_LBM_PERIODIC) NB_FAIL(NB_EINVAL, "bad bc");
    nb_grid *g = fin->g;
    cudaSetDevice(g->device);
    if (g->sparse) return sp_lbm_step(pfin, pfout, prm, nsteps);
    const bool per = prm->bc == NB_LBM_PERIODIC;
    const bool dist = nb_halo_on_stream(g);  // halos on the halo stream (NCCL or device copies)
    // make fin's halos current (covers states written by upload/init)
    NB_TRY(lbm_halo(fin, per, g->cs));
    HaloSync hs;
    if (dist) {
        NB_CUDA(cudaEventCreateWithFlags(&hs.eb, cudaEventDisableTiming));
        NB_CUDA(cudaEventCreateWithFlags(&hs.eh, cudaEventDisableTiming));
    }
    nb_status st = NB_OK;
    for (int t = 0; t < nsteps && st == NB_OK; ++t) {
        // boundary planes first (their outputs are the next step's halos)
        for (int p = g->first_local; p < g->first_local + g->nlocal && st == NB_OK; ++p) {
            int nz = g->parts[p].nz();
            bool blo = lbm_lo(g, p, per) >= 0, bhi = lbm_hi(g, p, per) >= 0;
            if (occ == NB_OCC_NONE || (!blo && !bhi)) {
                st = launch_lbm(g, p, fin, fout, prm, 0, nz, !dist);
            } else {
                if (blo) st = launch_lbm(g, p, fin, fout, prm, 0, 1, !dist);
                if (st == NB_OK && bhi && !(blo && nz == 1)) st = launch_lbm(g, p, fin, fout, prm, nz - 1, nz, !dist);
            }
        }
        if (st != NB_OK) break;
        // the halo stream starts after the boundary planes (event eb); the
        // interior kernels are ENQUEUED before the halo transfer so the host
        // never holds them back behind the transfer's API calls
        if (dist) cudaEventRecord(hs.eb, g->cs);
        // peer transport: the boundary kernels stored the halos into the
        // neighbours' fout; tell them (their wait follows their interior)
        if (st == NB_OK && nb_is_peer(g)) st = nb_peer_signal(g, per, g->cs);
        for (int p = g->first_local; p < g->first_local + g->nlocal && st == NB_OK; ++p) {
            int nz = g->parts[p].nz();
            bool blo = lbm_lo(g, p, per) >= 0, bhi = lbm_hi(g, p, per) >= 0;
            if (occ == NB_OCC_NONE || (!blo && !bhi)) continue;
            st = launch_lbm(g, p, fin, fout, prm, blo ? 1 : 0, bhi ? nz - 1 : nz, false);
        }
        if (dist && st == NB_OK) {  // halos on the halo stream, overlapped with the interior
            cudaStreamWaitEvent(g->hs, hs.eb, 0);
            st = lbm_halo(fout, per, g->hs);
            cudaEventRecord(hs.eh, g->hs);
            cudaStreamWaitEvent(g->cs, hs.eh, 0);
        }
        if (st == NB_OK && nb_is_peer(g)) st = nb_peer_wait(g, per, g->cs);
        std::swap(fin, fout);
    }
    if (hs.eb) {
        cudaEventDestroy(hs.eb);
        cudaEventDestroy(hs.eh);
    }
    *pfin = fin;
    *pfout = fout;
    return st;
}

// ===========================================================================
// AA pattern (PAPER.md L451 stlbm's AA / twoPop / Swap
// variants): ONE population buffer, updated in place — half the memory of
// twoPop, so twice the domain per GPU.  With P_t = twoPop's post-collision
// populations (natural layout A[x][i] = P_t(x, i) at even times):
//   even step: f_i = A[x - c_i][i]            (wall: A[x][opp(i)] + lid_i)
//              collide -> o;  A[x + c_i][opp(i)] = o_i
//                             (wall: A[x][i] = o_i + lid_opp(i))
//   odd step:  f_i = A[x][opp(i)];  collide -> o;  A[x][i] = o_i  (local)
// Every (location, slot) is read and written by one cell only, so the
// update is race free in place.  The gathered values are exactly twoPop's
// and the collision is shared, so 2k AA steps equal 2k twoPop steps bit for
// bit.  Partitions: the even step needs twoPop's halo (c_z = +1 populations
// up, -1 down) and stores the populations leaving the slab straight into
// the neighbour's own boundary plane (reversed slots); the odd step is
// local.
// ===========================================================================
struct LbmAAArgs {
    float *f[Q19];       // component base pointers (plane zl = -1, row 0)
    float *up[Q19];      // upper neighbour's components at its plane 0 (14..18 written)
    float *dn[Q19];      // lower neighbour's components at its top plane (9..13 written)
    PGeo g;
    float omega, ulid, rho_w;
};

template <bool EVEN, bool PERIODIC>
#ifndef NB_AA_BX
#define NB_AA_BX 32
#endif
#ifndef NB_AA_MINB
// 28 CTAs of one warp per SM (<= 73 registers): 3.49 against 3.95 ms/step
// with the unconstrained 95 registers (24: 3.66, 32: 3.50; tools/aa_ab.sh)
#define NB_AA_MINB 28
#endif
__global__ void __launch_bounds__(NB_AA_BX, NB_AA_MINB) k_lbm_aa(LbmAAArgs A) {  // 32 wide: 3.44 ms/step at 512^3 (64: 3.62, 128: 3.69, 256: 4.0)
    const int x = blockIdx.x * blockDim.x + threadIdx.x;
    const int y = blockIdx.y;
    const int zl = blockIdx.z;
    const PGeo &g = A.g;
    if (x >= g.nx) return;
    const int gz = g.z0 + zl;
    const int64_t row = (int64_t)y * g.pitch + x;
    const int64_t cell = (int64_t)(zl + 1) * g.ps + row;
    float f[Q19], o[Q19];
    if (!EVEN) {  // local: reversed slots in, natural slots out
#pragma unroll
        for (int i = 0; i < Q19; ++i) f[i] = __ldg(A.f[OPPv(i)] + cell);
        lbm_collide(f, A.omega, o);
#pragma unroll
        for (int i = 0; i < Q19; ++i) __stcs(A.f[i] + cell, o[i]);
        return;
    }
    // even, interior cell (every source and target inside the slab): 19
    // independent loads and 19 stores at uniform offsets
    if (x > 0 && x < g.nx - 1 && y > 0 && y < g.ny - 1 && zl > 0 && zl < g.nzl - 1) {
#pragma unroll
        for (int i = 0; i < Q19; ++i)
            f[i] = __ldg(A.f[i] + cell - (int64_t)CZv(i) * g.ps - (int64_t)CYv(i) * g.pitch - CXv(i));
        lbm_collide(f, A.omega, o);
#pragma unroll
        for (int i = 0; i < Q19; ++i)
            __stcs(A.f[OPPv(i)] + cell + (int64_t)CZv(i) * g.ps + (int64_t)CYv(i) * g.pitch + CXv(i), o[i]);
        return;
    }
    // even: twoPop's pull gather from the natural layout
#pragma unroll
    for (int i = 0; i < Q19; ++i) {
        int sx = x - CXv(i), sy = y - CYv(i);
        const int szl = zl - CZv(i), sgz = gz - CZv(i);
        if (PERIODIC) {
            sx = sx < 0 ? sx + g.nx : (sx >= g.nx ? sx - g.nx : sx);
            sy = sy < 0 ? sy + g.ny : (sy >= g.ny ? sy - g.ny : sy);
            f[i] = __ldg(A.f[i] + (int64_t)(szl + 1) * g.ps + (int64_t)sy * g.pitch + sx);
        } else {
            const bool inside = sx >= 0 && sx < g.nx && sy >= 0 && sy < g.ny && sgz >= 0 && sgz < g.NZ;
            float v = __ldg(inside ? A.f[i] + (int64_t)(szl + 1) * g.ps + (int64_t)sy * g.pitch + sx
                                   : A.f[OPPv(i)] + cell);
            if (CXv(i) != 0 && sy == g.ny && sx >= 0 && sx < g.nx && sgz >= 0 && sgz < g.NZ)
                v = v + 6.0f * Wv(i) * A.rho_w * ((float)CXv(i) * A.ulid);
            f[i] = v;
        }
    }
    lbm_collide(f, A.omega, o);
    // push o_i to x + c_i, reversed slot; a wall reflects it into this cell
#pragma unroll
    for (int i = 0; i < Q19; ++i) {
        int tx = x + CXv(i), ty = y + CYv(i);
        const int tzl = zl + CZv(i), tgz = gz + CZv(i);
        const int j = OPPv(i);
        if (!PERIODIC && !(tx >= 0 && tx < g.nx && ty >= 0 && ty < g.ny && tgz >= 0 && tgz < g.NZ)) {
            float v = o[i];  // read next step as population j of this cell (twoPop's bounce-back)
            if (CXv(j) != 0 && ty == g.ny && tx >= 0 && tx < g.nx && tgz >= 0 && tgz < g.NZ)
                v = v + 6.0f * Wv(j) * A.rho_w * ((float)CXv(j) * A.ulid);
            A.f[i][cell] = v;
            continue;
        }
        if (PERIODIC) {
            tx = tx < 0 ? tx + g.nx : (tx >= g.nx ? tx - g.nx : tx);
            ty = ty < 0 ? ty + g.ny : (ty >= g.ny ? ty - g.ny : ty);
        }
        const int64_t trow = (int64_t)ty * g.pitch + tx;
        if (tzl >= 0 && tzl < g.nzl)
            A.f[j][(int64_t)(tzl + 1) * g.ps + trow] = o[i];
        else if (tzl == g.nzl)
            A.up[j][trow] = o[i];  // upper neighbour's plane 0
        else
            A.dn[j][trow] = o[i];  // lower neighbour's top plane
    }
}

extern "C" nb_status nb_lbm_step_aa(nb_field *f, const nb_lbm_params *prm, int32_t nsteps) {
    if (!f || !prm) NB_FAIL(NB_EINVAL, "nb_lbm_step_aa: NULL argument");
    NB_TRY(lbm_check(f));
    if (nsteps < 0 || (nsteps & 1)) NB_FAIL(NB_EINVAL, "nb_lbm_step_aa: nsteps must be even (got %d)", nsteps);
    NB_LAYOUTS(f, 1 << NB_SOA, "nb_lbm_step_aa");
    if (prm->bc != NB_LBM_CAVITY && prm->bc != NB_LBM_PERIODIC) NB_FAIL(NB_EINVAL, "bad bc");
    nb_grid *g = f->g;
    if (g->sparse) NB_FAIL(NB_EUNSUPPORTED, "AA pattern on element-sparse grids is not built");
    if (nb_halo_on_stream(g)) NB_FAIL(NB_EUNSUPPORTED, "AA pattern: fused (in-process / peer) halos only");
    cudaSetDevice(g->device);
    const bool per = prm->bc == NB_LBM_PERIODIC;
    for (int t = 0; t < nsteps; ++t) {
        const bool even = !(t & 1);
        if (even) NB_TRY(nb_halo_run(f, per, 9, 14, 14, 19, g->cs));  // twoPop's halo: the pull sources
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            LbmAAArgs A;
            memset(&A, 0, sizeof(A));
            for (int i = 0; i < Q19; ++i) A.f[i] = (float *)f->base[p] + (int64_t)i * lcs(f, p);
            A.g = pgeo(f, p);
            A.omega = (float)prm->omega;
            A.ulid = (float)prm->u_lid;
            A.rho_w = (float)prm->rho_w;
            const int lo = lbm_lo(g, p, per), hi = lbm_hi(g, p, per);
            if (even) {
                if (hi >= 0) {
                    if (!nb_reachable(f, hi)) NB_FAIL(NB_EUNSUPPORTED, "AA pattern: neighbour not addressable");
                    for (int i = 14; i < 19; ++i)
                        A.up[i] = (float *)f->base[hi] + (int64_t)i * lcs(f, hi) + (int64_t)1 * f->ps;
                }
                if (lo >= 0) {
                    if (!nb_reachable(f, lo)) NB_FAIL(NB_EUNSUPPORTED, "AA pattern: neighbour not addressable");
                    for (int i = 9; i < 14; ++i)
                        A.dn[i] = (float *)f->base[lo] + (int64_t)i * lcs(f, lo) + (int64_t)g->parts[lo].nz() * f->ps;
                }
            }
            dim3 blk(NB_AA_BX), grd((g->nx + NB_AA_BX - 1) / NB_AA_BX, g->ny, A.g.nzl);
            LaunchScope ls(g, g->cs, "k_lbm_aa");
            if (even)
                per ? k_lbm_aa<true, true><<<grd, blk, 0, g->cs>>>(A) : k_lbm_aa<true, false><<<grd, blk, 0, g->cs>>>(A);
            else
                per ? k_lbm_aa<false, true><<<grd, blk, 0, g->cs>>>(A)
                    : k_lbm_aa<false, false><<<grd, blk, 0, g->cs>>>(A);
            NB_TRY(nb_launch_check("k_lbm_aa"));
        }
        // peer transport: the even step stored into the neighbours' planes
        if (even && nb_is_peer(g)) NB_TRY(nb_peer_round(g, per, g->cs));
    }
    return NB_OK;
}

extern "C" nb_status nb_lbm_macroscopic(const nb_field *f, nb_field *rho, nb_field *u) {
    NB_TRY(lbm_check(f));
    if (!rho || !u) NB_FAIL(NB_EINVAL, "NULL field");
    if (rho->g != f->g || u->g != f->g) NB_FAIL(NB_EMISMATCH, "fields belong to different grids");
    if (rho->dt != NB_F32 || u->dt != NB_F32 || rho->card != 1 || u->card != 3)
        NB_FAIL(NB_EMISMATCH, "rho: fp32 card 1, u: fp32 card 3");
    nb_grid *g = f->g;
    cudaSetDevice(g->device);
    if (g->sparse) {
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            const NbSparsePart &sp = g->sp[p];
            if (sp.n == 0) continue;
            LaunchScope ls(g, g->cs, "k_lbm_macro");
            k_sp_lbm_macro<<<(unsigned)((sp.n + 127) / 128), 128, 0, g->cs>>>(
                (const float *)f->base[p], (float *)rho->base[p], (float *)u->base[p], f->pcs[p], rho->pcs[p],
                u->pcs[p], sp.hl, sp.n);
            NB_TRY(nb_launch_check("k_sp_lbm_macro"));
        }
        return NB_OK;
    }
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        PGeo geo = pgeo(f, p);
        dim3 blk(128), grd((g->nx + 127) / 128, g->ny, geo.nzl);
        LaunchScope ls(g, g->cs, "k_lbm_macro");
        k_lbm_macro<<<grd, blk, 0, g->cs>>>((const float *)f->base[p], (float *)rho->base[p], (float *)u->base[p], geo,
                                            LbmFa{f->ps, lcs(f, p), f->es}, LbmFa{rho->ps, lcs(rho, p), rho->es},
                                            LbmFa{u->ps, lcs(u, p), u->es});
        NB_TRY(nb_launch_check("k_lbm_macro"));
    }
    return NB_OK;
}
