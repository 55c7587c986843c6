// nb_sparse.cu — element-sparse grid ("element-sparse, where
// only cells of interest are stored with their connectivity table"; L256:
// boundary cells in contiguous segments, two transfers per partition, no
// marshalling; L472: dense vs sparse trade-off).  SURVEY.md §8(a) a9.
//
// Layout per partition and component: [halo_lo | own | halo_hi] where own =
// the slab's active cells in (z, y, x) order, halo_lo / halo_hi = the active
// cells of the neighbours' adjacent planes in (y, x) order.  The connectivity
// table conn[d][j] (d = -x, +x, -y, +y, -z, +z) holds the buffer index of the
// neighbour of own cell j, or -1 for an inactive / out-of-domain neighbour
// (read as outside).  Built on the device: an exclusive scan (CUB) of the
// slab mask numbers the active cells directly in buffer order.
//
// Canonical dot order (sparse): per plane (c, z), the plane's active cells
// in (y, x) order are cut into 256-cell segments; a segment is reduced by
// xor-butterflies over warps then the 8 warps in order; segment values, then
// plane sums, by the fixed block tree of nb_reduce_finalize.  Independent of
// the partitioning (a plane's cells and their order do not depend on it).
#include <cub/device/device_scan.cuh>
#include <cub/iterator/transform_input_iterator.cuh>

#include <algorithm>
#include <vector>

#include "nb_device.cuh"
#include "nb_internal.cuh"

constexpr int SEG = 256;

std::vector<std::pair<int, int>> view_ranges(const nb_grid *g, int p, nb_view v);

namespace {
struct MaskToInt {
    __host__ __device__ int operator()(uint8_t v) const { return v ? 1 : 0; }
};
}  // namespace

void nb_sparse_free(nb_grid *g) {
    for (auto &s : g->sp) {
        cudaFree(s.conn);
        cudaFree(s.conn19);
        s.conn19 = nullptr;
        cudaFree(s.coord);
        cudaFree(s.d_pstart);
        cudaFree(s.d_seg);
        cudaFree(s.d_seg_bnd);
        cudaFree(s.d_seg_bnd_gi);
        cudaFree(s.d_nbr);
        cudaFree(s.d_seginfo);
        cudaFree(s.d_fm);
        cudaFree(s.d_fb);
        s.d_fm = nullptr;
        s.d_fb = nullptr;
        cudaFree(s.d_rm);
        cudaFree(s.d_ri);
        s.d_rm = nullptr;
        s.d_ri = nullptr;
        s.tile_any.clear();
        cudaFree(s.d_fnode);
        s.d_fnode = nullptr;
        s.fnode_start.clear();
        for (auto &kv : s.box_lists) cudaFree(kv.second.first);
        s.box_lists.clear();
        s.d_seg_bnd = s.d_seg_bnd_gi = nullptr;
        s.d_nbr = s.d_seginfo = nullptr;
        s.n_runs = 0;
        s.n_seg_bnd = -1;
        s.conn = s.coord = nullptr;
        s.d_pstart = nullptr;
        s.d_seg = nullptr;
    }
}

__global__ void k_sp_conn(const uint8_t *__restrict__ mask, const int32_t *__restrict__ map, int nx, int ny,
                          int slab_z0, int nslab, int z0, int NZ, int hl, int64_t n, int32_t *conn, int32_t *coord) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y, z = z0 + blockIdx.z;
    if (x >= nx) return;
    const int64_t plane = (int64_t)nx * ny;
    const int64_t cell = (int64_t)(z - slab_z0) * plane + (int64_t)y * nx + x;
    if (!mask[cell]) return;
    const int64_t j = (int64_t)map[cell] - hl;
    coord[j] = x | (y << 16);
    const int dx[6] = {-1, 1, 0, 0, 0, 0}, dy[6] = {0, 0, -1, 1, 0, 0}, dz[6] = {0, 0, 0, 0, -1, 1};
#pragma unroll
    for (int d = 0; d < 6; ++d) {
        int xx = x + dx[d], yy = y + dy[d], zz = z + dz[d];
        int32_t v = -1;
        if (xx >= 0 && xx < nx && yy >= 0 && yy < ny && zz >= 0 && zz < NZ && zz - slab_z0 >= 0 &&
            zz - slab_z0 < nslab) {
            int64_t nc = (int64_t)(zz - slab_z0) * plane + (int64_t)yy * nx + xx;
            if (mask[nc]) v = map[nc];
        }
        conn[(int64_t)d * n + j] = v;
    }
}

static nb_status sp_bnd_segments(nb_grid *g, int p);
static nb_status sp_build_runs(nb_grid *g, int p);

extern "C" nb_status nb_grid_create_sparse(const int32_t dims[3], const uint8_t *active, int32_t nparts,
                                           const int32_t *device_ids, nb_comm *comm, nb_grid **out) {
    if (!out || !dims || !active) NB_FAIL(NB_EINVAL, "nb_grid_create_sparse: NULL argument");
    *out = nullptr;
    if (dims[0] < 1 || dims[1] < 1 || dims[2] < 1 || dims[0] > 65535 || dims[1] > 32767)
        NB_FAIL(NB_EINVAL, "nb_grid_create_sparse: bad dims");
    const int nx = dims[0], ny = dims[1], nz = dims[2];
    const int64_t plane = (int64_t)nx * ny;
    std::vector<int64_t> counts(nz, 0);
    for (int z = 0; z < nz; ++z) {
        const uint8_t *m = active + z * plane;
        int64_t c = 0;
        for (int64_t i = 0; i < plane; ++i) c += m[i] != 0;
        counts[z] = c;
    }
    if (nparts < 1 || nparts > nz) NB_FAIL(NB_EINVAL, "nb_grid_create_sparse: bad nparts %d", nparts);
    // segment entries are int32 (zl << 16 | k) with -1 as the sentinel: zl <= 32767 keeps them >= 0
    if (nz > 32767 || plane > (int64_t)SEG * 65535)
        NB_FAIL(NB_EUNSUPPORTED, "nb_grid_create_sparse: segment table limits (nz <= 32767, Nx*Ny <= 16.7M)");
    std::vector<int32_t> zb(nparts + 1);
    NB_TRY(nb_partition_plan_weighted(nz, counts.data(), nparts, zb.data()));
    if (nparts > 1)
        for (int p = 0; p < nparts; ++p)
            if (zb[p + 1] - zb[p] < 2) NB_FAIL(NB_EUNSUPPORTED, "sparse slab %d has < 2 planes", p);
    nb_grid *g = new nb_grid();
    g->sparse = true;
    g->nx = nx;
    g->ny = ny;
    g->nz = nz;
    g->plane_count = counts;
    g->host_mask.assign(active, active + (size_t)nz * plane);
    int64_t maxc = 1;
    for (auto c : counts) {
        g->n_active += c;
        maxc = std::max(maxc, c);
    }
    g->T = (int)((maxc + SEG - 1) / SEG);
    nb_status s = nb_grid_setup_parts(g, zb.data(), nparts, device_ids, comm);
    if (s == NB_OK) s = nb_grid_alloc_common(g);
    if (s != NB_OK) {
        nb_grid_destroy(g);
        return s;
    }
    g->sp.resize(nparts);
    int64_t a0 = 0;
    for (int p = 0; p < nparts; ++p) {
        NbPart &q = g->parts[p];
        q.a0 = a0;
        q.n_act = 0;
        for (int z = q.z0; z < q.z1; ++z) q.n_act += counts[z];
        a0 += q.n_act;
        q.n_lo_bnd = q.lo >= 0 ? counts[q.z0] : 0;
        q.n_hi_bnd = q.hi >= 0 ? counts[q.z1 - 1] : 0;
        q.halo_lo = q.lo >= 0 ? counts[q.z0 - 1] : 0;
        q.halo_hi = q.hi >= 0 ? counts[q.z1] : 0;
        NbSparsePart &sp = g->sp[p];
        sp.hl = q.halo_lo;
        sp.n = q.n_act;
        sp.hh = q.halo_hi;
        sp.cs = std::max<int64_t>(32, (sp.hl + sp.n + sp.hh + 31) / 32 * 32);
        sp.pstart.assign(q.nz() + 1, 0);
        sp.seg_start.assign(q.nz() + 1, 0);
        for (int z = q.z0; z < q.z1; ++z) {
            sp.pstart[z - q.z0 + 1] = sp.pstart[z - q.z0] + counts[z];
            sp.seg_start[z - q.z0 + 1] = sp.seg_start[z - q.z0] + (counts[z] + SEG - 1) / SEG;
            sp.max_plane = std::max<int>(sp.max_plane, (int)counts[z]);
        }
    }
    cudaSetDevice(g->device);
    for (int p = g->first_local; p < g->first_local + g->nlocal && s == NB_OK; ++p) {
        NbPart &q = g->parts[p];
        NbSparsePart &sp = g->sp[p];
        const int slab_z0 = q.z0 - (q.lo >= 0 ? 1 : 0), slab_z1 = q.z1 + (q.hi >= 0 ? 1 : 0);
        const int nslab = slab_z1 - slab_z0;
        const int64_t ncell = (int64_t)nslab * plane;
        uint8_t *d_mask = nullptr;
        int32_t *d_map = nullptr;
        void *tmp = nullptr;
        size_t tmp_bytes = 0;
        auto fail = [&](const char *what, cudaError_t e) {
            nb_set_error("nb_grid_create_sparse: %s: %s", what, cudaGetErrorString(e));
            s = NB_ECUDA;
        };
        cudaError_t e;
        if ((e = cudaMalloc(&d_mask, ncell)) != cudaSuccess) fail("cudaMalloc mask", e);
        if (s == NB_OK && (e = cudaMalloc(&d_map, ncell * 4)) != cudaSuccess) fail("cudaMalloc map", e);
        if (s == NB_OK && (e = cudaMemcpyAsync(d_mask, active + (int64_t)slab_z0 * plane, ncell,
                                               cudaMemcpyHostToDevice, g->cs)) != cudaSuccess)
            fail("mask upload", e);
        cub::TransformInputIterator<int, MaskToInt, const uint8_t *> it(d_mask, MaskToInt());
        if (s == NB_OK) {
            cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, it, d_map, ncell, g->cs);
            if ((e = cudaMalloc(&tmp, tmp_bytes)) != cudaSuccess) fail("cudaMalloc scan temp", e);
        }
        if (s == NB_OK && (e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, it, d_map, ncell, g->cs)) != cudaSuccess)
            fail("scan", e);
        if (s == NB_OK && (e = cudaMalloc(&sp.conn, sizeof(int32_t) * 6 * std::max<int64_t>(sp.n, 1))) != cudaSuccess)
            fail("cudaMalloc conn", e);
        if (s == NB_OK && (e = cudaMalloc(&sp.coord, sizeof(int32_t) * std::max<int64_t>(sp.n, 1))) != cudaSuccess)
            fail("cudaMalloc coord", e);
        if (s == NB_OK && (e = cudaMalloc(&sp.d_pstart, sizeof(int64_t) * sp.pstart.size())) != cudaSuccess)
            fail("cudaMalloc pstart", e);
        if (s == NB_OK)
            cudaMemcpyAsync(sp.d_pstart, sp.pstart.data(), sizeof(int64_t) * sp.pstart.size(), cudaMemcpyHostToDevice,
                            g->cs);
        std::vector<int32_t> segs;
        for (int zl = 0; zl < q.nz(); ++zl)
            for (int64_t k = 0; k < sp.seg_start[zl + 1] - sp.seg_start[zl]; ++k) segs.push_back((zl << 16) | (int)k);
        if (s == NB_OK && (e = cudaMalloc(&sp.d_seg, sizeof(int32_t) * std::max<size_t>(segs.size(), 1))) != cudaSuccess)
            fail("cudaMalloc seg", e);
        if (s == NB_OK && !segs.empty())
            cudaMemcpyAsync(sp.d_seg, segs.data(), sizeof(int32_t) * segs.size(), cudaMemcpyHostToDevice, g->cs);
        if (s == NB_OK) s = sp_bnd_segments(g, p);  // built here: the CG hooks may run under graph capture
        if (s == NB_OK) s = sp_build_runs(g, p);
        if (s == NB_OK && q.nz() > 0) {
            dim3 blk(128), grd((nx + 127) / 128, ny, q.nz());
            LaunchScope ls(g, g->cs, "k_sp_conn");
            k_sp_conn<<<grd, blk, 0, g->cs>>>(d_mask, d_map, nx, ny, slab_z0, nslab, q.z0, nz, (int)sp.hl, sp.n,
                                              sp.conn, sp.coord);
            s = nb_launch_check("k_sp_conn");
        }
        cudaStreamSynchronize(g->cs);
        cudaFree(d_mask);
        cudaFree(d_map);
        cudaFree(tmp);
    }
    if (s != NB_OK) {
        nb_grid_destroy(g);
        return s;
    }
    *out = g;
    return NB_OK;
}

// ---------------------------------------------------------------------------
// fields
// ---------------------------------------------------------------------------
template <typename T>
__global__ void k_sp_fill_const(T *p, int64_t n, T v) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = v;
}

nb_status nb_sparse_field_alloc(nb_field *f) {
    nb_grid *g = f->g;
    f->pcs.assign(g->nparts, 0);
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbSparsePart &sp = g->sp[p];
        f->pcs[p] = sp.cs;
        size_t bytes = (size_t)sp.cs * f->card * f->esz;
        NB_TRY(nb_field_buf_alloc(g, bytes, (void **)&f->base[p]));
        f->bytes[p] = bytes;
        if (f->outside == 0.0) {
            NB_CUDA(cudaMemsetAsync(f->base[p], 0, bytes, g->cs));
        } else {
            int64_t n = (int64_t)(bytes / f->esz);
            LaunchScope ls(g, g->cs, "k_fill_const");
            if (f->dt == NB_F64)
                k_sp_fill_const<double><<<296, 256, 0, g->cs>>>((double *)f->base[p], n, f->outside);
            else
                k_sp_fill_const<float><<<296, 256, 0, g->cs>>>((float *)f->base[p], n, (float)f->outside);
            NB_TRY(nb_launch_check("k_fill_const"));
        }
    }
    f->cs = f->pcs[g->first_local];
    return NB_OK;
}

// plane-organised launch over own slots: grid (segments, planes), 256 threads
static dim3 sp_grid(const NbSparsePart &sp, int nplanes) {
    return dim3((unsigned)std::max(1, (sp.max_plane + SEG - 1) / SEG), (unsigned)std::max(1, nplanes));
}

// gather / scatter between a dense slab [z][y][x] and the own region
template <typename T>
__global__ void k_sp_gather(const T *__restrict__ dense, T *__restrict__ own, const int32_t *coord,
                            const int64_t *pstart, int nx, int ny, int zb) {
    const int zl = zb + blockIdx.y;
    const int64_t j = pstart[zl] + (int64_t)blockIdx.x * SEG + threadIdx.x;
    if (j >= pstart[zl + 1]) return;
    const int c = coord[j], x = c & 0xffff, y = c >> 16;
    own[j] = dense[((int64_t)zl * ny + y) * nx + x];
}

template <typename T>
__global__ void k_sp_scatter(T *__restrict__ dense, const T *__restrict__ own, const int32_t *coord,
                             const int64_t *pstart, int nx, int ny, int zb) {
    const int zl = zb + blockIdx.y;
    const int64_t j = pstart[zl] + (int64_t)blockIdx.x * SEG + threadIdx.x;
    if (j >= pstart[zl + 1]) return;
    const int c = coord[j], x = c & 0xffff, y = c >> 16;
    dense[((int64_t)zl * ny + y) * nx + x] = own[j];
}

nb_status nb_sparse_upload(nb_field *f, const void *host) {
    nb_grid *g = f->g;
    const int64_t plane = (int64_t)g->nx * g->ny;
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbPart &q = g->parts[p];
        const NbSparsePart &sp = g->sp[p];
        size_t slab = (size_t)plane * q.nz() * f->esz;
        void *tmp = nullptr;
        NB_CUDA(cudaMallocAsync(&tmp, std::max<size_t>(slab, 1), g->cs));
        for (int c = 0; c < f->card; ++c) {
            const char *src = (const char *)host + ((size_t)c * g->nz + q.z0) * plane * f->esz;
            NB_CUDA(cudaMemcpyAsync(tmp, src, slab, cudaMemcpyHostToDevice, g->cs));
            char *own = f->base[p] + ((int64_t)c * sp.cs + sp.hl) * f->esz;
            LaunchScope ls(g, g->cs, "k_sp_gather");
            if (f->dt == NB_F64)
                k_sp_gather<double><<<sp_grid(sp, q.nz()), SEG, 0, g->cs>>>((const double *)tmp, (double *)own, sp.coord,
                                                                            sp.d_pstart, g->nx, g->ny, 0);
            else
                k_sp_gather<float><<<sp_grid(sp, q.nz()), SEG, 0, g->cs>>>((const float *)tmp, (float *)own, sp.coord,
                                                                           sp.d_pstart, g->nx, g->ny, 0);
            NB_TRY(nb_launch_check("k_sp_gather"));
        }
        NB_CUDA(cudaFreeAsync(tmp, g->cs));
    }
    NB_CUDA(cudaStreamSynchronize(g->cs));
    return NB_OK;
}

nb_status nb_sparse_download(const nb_field *f, void *host) {
    nb_grid *g = f->g;
    const int64_t plane = (int64_t)g->nx * g->ny;
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbPart &q = g->parts[p];
        const NbSparsePart &sp = g->sp[p];
        size_t slab = (size_t)plane * q.nz() * f->esz;
        void *tmp = nullptr;
        NB_CUDA(cudaMallocAsync(&tmp, std::max<size_t>(slab, 1), g->cs));
        for (int c = 0; c < f->card; ++c) {
            int64_t n = (int64_t)(slab / f->esz);
            {
                LaunchScope ls(g, g->cs, "k_fill_const");
                if (f->dt == NB_F64)
                    k_sp_fill_const<double><<<296, 256, 0, g->cs>>>((double *)tmp, n, f->outside);
                else
                    k_sp_fill_const<float><<<296, 256, 0, g->cs>>>((float *)tmp, n, (float)f->outside);
            }
            const char *own = f->base[p] + ((int64_t)c * sp.cs + sp.hl) * f->esz;
            LaunchScope ls(g, g->cs, "k_sp_scatter");
            if (f->dt == NB_F64)
                k_sp_scatter<double><<<sp_grid(sp, q.nz()), SEG, 0, g->cs>>>((double *)tmp, (const double *)own,
                                                                             sp.coord, sp.d_pstart, g->nx, g->ny, 0);
            else
                k_sp_scatter<float><<<sp_grid(sp, q.nz()), SEG, 0, g->cs>>>((float *)tmp, (const float *)own, sp.coord,
                                                                            sp.d_pstart, g->nx, g->ny, 0);
            NB_TRY(nb_launch_check("k_sp_scatter"));
            char *dst = (char *)host + ((size_t)c * g->nz + q.z0) * plane * f->esz;
            NB_CUDA(cudaMemcpyAsync(dst, tmp, slab, cudaMemcpyDeviceToHost, g->cs));
        }
        NB_CUDA(cudaFreeAsync(tmp, g->cs));
    }
    NB_CUDA(cudaStreamSynchronize(g->cs));
    return NB_OK;
}

template <typename T>
__global__ void k_sp_fill(T *own, const int32_t *coord, const int64_t *pstart, int z0, int nx, int ny, int NZ,
                          int nzp, int64_t cs, int kind, uint64_t seed, double a, double b, double h) {
    const int zl = blockIdx.y % nzp, c = blockIdx.y / nzp;
    const int64_t j = pstart[zl] + (int64_t)blockIdx.x * SEG + threadIdx.x;
    if (j >= pstart[zl + 1]) return;
    const int cc = coord[j], x = cc & 0xffff, y = cc >> 16, z = z0 + zl;
    uint64_t gidx = (uint64_t)x + (uint64_t)nx * ((uint64_t)y + (uint64_t)ny * ((uint64_t)z + (uint64_t)NZ * c));
    own[(int64_t)c * cs + j] = (T)nb_gen(kind, seed, gidx, a, b, x, y, z, h);
}

nb_status nb_sparse_fill(nb_field *f, nb_fill kind, uint64_t seed, double a, double b) {
    nb_grid *g = f->g;
    double h = 1.0 / (double)(g->nx + 1);
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbPart &q = g->parts[p];
        const NbSparsePart &sp = g->sp[p];
        if (q.nz() == 0) continue;
        dim3 grd = sp_grid(sp, q.nz() * f->card);
        LaunchScope ls(g, g->cs, "k_sp_fill");
        if (f->dt == NB_F64)
            k_sp_fill<double><<<grd, SEG, 0, g->cs>>>((double *)f->base[p] + sp.hl, sp.coord, sp.d_pstart, q.z0, g->nx,
                                                      g->ny, g->nz, q.nz(), sp.cs, kind, seed, a, b, h);
        else
            k_sp_fill<float><<<grd, SEG, 0, g->cs>>>((float *)f->base[p] + sp.hl, sp.coord, sp.d_pstart, q.z0, g->nx,
                                                     g->ny, g->nz, q.nz(), sp.cs, kind, seed, a, b, h);
        NB_TRY(nb_launch_check("k_sp_fill"));
    }
    return NB_OK;
}

// The compact index of partition p's slab with its halo planes (the map
// nb_grid_create_sparse builds the connectivity from): device mask and
// exclusive-scan map of planes [slab_z0, slab_z0 + nslab); caller frees.
nb_status nb_sparse_slab_map(nb_grid *g, int p, uint8_t **d_mask, int32_t **d_map, int *slab_z0, int *nslab) {
    const NbPart &q = g->parts[p];
    const int64_t plane = (int64_t)g->nx * g->ny;
    *slab_z0 = q.z0 - (q.lo >= 0 ? 1 : 0);
    *nslab = q.z1 + (q.hi >= 0 ? 1 : 0) - *slab_z0;
    const int64_t ncell = (int64_t)*nslab * plane;
    *d_mask = nullptr;
    *d_map = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    NB_CUDA(cudaMalloc(d_mask, ncell));
    NB_CUDA(cudaMalloc(d_map, ncell * 4));
    NB_CUDA(cudaMemcpyAsync(*d_mask, g->host_mask.data() + (int64_t)*slab_z0 * plane, ncell, cudaMemcpyHostToDevice,
                            g->cs));
    cub::TransformInputIterator<int, MaskToInt, const uint8_t *> it(*d_mask, MaskToInt());
    NB_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, it, *d_map, ncell, g->cs));
    NB_CUDA(cudaMalloc(&tmp, tmp_bytes));
    NB_CUDA(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, it, *d_map, ncell, g->cs));
    NB_CUDA(cudaStreamSynchronize(g->cs));
    cudaFree(tmp);
    return NB_OK;
}

// ---------------------------------------------------------------------------
// halo: contiguous segments (the neighbour's adjacent plane), plan order
// ---------------------------------------------------------------------------
nb_status nb_sparse_halo_comps(nb_field *f, int c0u, int c1u, int c0d, int c1d);
nb_status nb_sparse_halo_update(nb_field *f) { return nb_sparse_halo_comps(f, 0, f->card, 0, f->card); }
nb_status nb_sparse_halo_comps(nb_field *f, int c0u, int c1u, int c0d, int c1d) {
    return nb_sparse_halo_run(f, c0u, c1u, c0d, c1d, f->g->cs, NB_HALO_GENERIC);
}

// components [c0u, c1u) travel up (last plane -> upper neighbour's low halo),
// [c0d, c1d) down; on stream s.  mode NB_HALO_GENERIC: with the peer
// transport a "ready" round before and a "done" round after the copies;
// NB_HALO_SEND: only the copies and a signal (the OCC split send of the CG
// schedules, whose reductions already order every halo read before the
// next write; the consumer calls nb_peer_wait)
nb_status nb_sparse_halo_run(nb_field *f, int c0u, int c1u, int c0d, int c1d, cudaStream_t s, int mode) {
    nb_grid *g = f->g;
    int world = g->comm ? g->comm->world : 1, rank = g->comm ? g->comm->rank : 0;
    int cnt = 0;
    NB_TRY(nb_halo_plan(g->nz, g->nparts, world, rank, 0, nullptr, 0, &cnt));
    std::vector<nb_halo_msg> msgs(cnt);
    NB_TRY(nb_halo_plan(g->nz, g->nparts, world, rank, 0, msgs.data(), cnt, &cnt));
    // message geometry from the sparse partitions (src segment, dst halo region)
    auto src_off = [&](const nb_halo_msg &m) -> int64_t {  // element offset in src buffer (component 0)
        const NbSparsePart &sp = g->sp[m.src_part];
        const NbPart &q = g->parts[m.src_part];
        return m.up ? sp.hl + sp.n - g->plane_count[q.z1 - 1] : sp.hl;
    };
    auto dst_off = [&](const nb_halo_msg &m) -> int64_t {
        const NbSparsePart &sp = g->sp[m.dst_part];
        return m.up ? 0 : sp.hl + sp.n;
    };
    auto count = [&](const nb_halo_msg &m) -> int64_t {
        const NbPart &q = g->parts[m.src_part];
        return g->plane_count[m.up ? q.z1 - 1 : q.z0];
    };
    // device-local segments, and with the peer transport every segment this
    // rank sends (into the neighbour's IPC-mapped halo), in one batched launch
    const bool peer = nb_is_peer(g);
    if (peer && mode == NB_HALO_GENERIC) NB_TRY(nb_peer_round(g, false, s));  // neighbours done reading these halos
    bool remote = false;
    CopyBatch cb;
    for (auto &m : msgs) {
        const bool mine = m.src_rank == rank && (peer || m.dst_rank == rank);
        const int c0 = m.up ? c0u : c0d, c1 = m.up ? c1u : c1d;
        if (mine) {
            for (int c = c0; c < c1 && count(m) > 0; ++c) {
                const char *src = f->base[m.src_part] + ((int64_t)c * f->pcs[m.src_part] + src_off(m)) * f->esz;
                char *dst = f->base[m.dst_part] + ((int64_t)c * f->pcs[m.dst_part] + dst_off(m)) * f->esz;
                if (cb.n == CopyBatch::MAX) {
                    NB_TRY(nb_launch_copy_batch(g, cb, s));
                    cb = CopyBatch();
                }
                cb.add(dst, src, count(m) * f->esz);
            }
        } else if (!(m.src_rank == rank && m.dst_rank == rank)) {
            remote = true;
        }
    }
    if (cb.n) NB_TRY(nb_launch_copy_batch(g, cb, s));
    if (peer) return mode == NB_HALO_GENERIC ? nb_peer_round(g, false, s) : nb_peer_signal(g, false, s);
    if (!remote) return NB_OK;
    NB_TRY(nb_nccl_group(g, true));
    for (auto &m : msgs) {
        if (m.src_rank == rank && m.dst_rank == rank) continue;
        if (count(m) == 0) continue;
        const int c0 = m.up ? c0u : c0d, c1 = m.up ? c1u : c1d;
        for (int c = c0; c < c1; ++c) {
            if (m.src_rank == rank)
                NB_TRY(nb_nccl_send(g, f->base[m.src_part] + ((int64_t)c * f->pcs[m.src_part] + src_off(m)) * f->esz,
                                    count(m) * f->esz, m.dst_rank, s));
            else
                NB_TRY(nb_nccl_recv(g, f->base[m.dst_part] + ((int64_t)c * f->pcs[m.dst_part] + dst_off(m)) * f->esz,
                                    count(m) * f->esz, m.src_rank, s));
        }
    }
    NB_TRY(nb_nccl_group(g, false));
    return NB_OK;
}

// ---------------------------------------------------------------------------
// maps (same per-element arithmetic as the dense k_axpby)
// ---------------------------------------------------------------------------
template <typename T>
__global__ void k_sp_axpby(const T *__restrict__ x, T *__restrict__ y, int64_t n, T a, T b, int mode) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        T xv = x[i];
        if (mode == 0)
            y[i] = a * xv;
        else if (mode == 1)
            y[i] = fma(a, xv, y[i]);
        else
            y[i] = fma(a, xv, b * y[i]);
    }
}

nb_status nb_sparse_axpby(double a, const nb_field *x, double b, nb_field *y, nb_view v) {
    nb_grid *g = x->g;
    int mode = (b == 0.0) ? 0 : (b == 1.0 ? 1 : 2);
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbSparsePart &sp = g->sp[p];
        for (auto rg : view_ranges(g, p, v)) {
            int64_t j0 = sp.pstart[rg.first], j1 = sp.pstart[rg.second];
            for (int c = 0; c < x->card; ++c) {
                int64_t off = (int64_t)c * sp.cs + sp.hl + j0, n = j1 - j0;
                if (n <= 0) continue;
                int blocks = (int)std::min<int64_t>((n + 255) / 256, 148 * 8);
                LaunchScope ls(g, g->cs, "k_sp_axpby");
                if (x->dt == NB_F64)
                    k_sp_axpby<double><<<blocks, 256, 0, g->cs>>>((const double *)x->base[p] + off,
                                                                  (double *)y->base[p] + off, n, a, b, mode);
                else
                    k_sp_axpby<float><<<blocks, 256, 0, g->cs>>>((const float *)x->base[p] + off,
                                                                 (float *)y->base[p] + off, n, (float)a, (float)b, mode);
                NB_TRY(nb_launch_check("k_sp_axpby"));
            }
        }
    }
    return NB_OK;
}

// ---------------------------------------------------------------------------
// plane-segment kernels: stencil / dot / CG phases.  Block = one 256-cell
// segment of one plane; the dot value of the segment is the canonical one.
// ---------------------------------------------------------------------------
enum { SPK_DOT = 0, SPK_LAP = 1, SPK_CG_INIT = 2, SPK_CG_MAP = 3, SPK_CG_Q = 4, SPK_CG_R = 5, SPK_CG_FLUSH = 6 };

struct SpArgs {
    const int32_t *seg;  // segment table of the partition
    int64_t seg0;        // first table entry of this launch
    int64_t nseg;        // table entries of this launch
    const int64_t *pstart;
    const int32_t *conn;
    int64_t n;       // own cells (conn stride)
    int64_t hl;      // own-region offset in the buffers
    int plane0;      // global plane index of local plane 0 (+ c*NZ)
    int T;
    double *tp;
    double outside;
    const double *a;  // kernel-specific operands (buffer base pointers)
    const double *b;
    double *c;
    double *d;
    CgScal *sc;
    int pf;         // k_sp_runs: L2 prefetch distance in blocks (0: none)
    float cps;      // k_sp_runs: mean cells per segment of the launch
};

template <typename T>
__device__ __forceinline__ T sp_nsum(const T *x, const int32_t *conn, int64_t n, int64_t j, T outside) {
    // canonical order -x, +x, -y, +y, -z, +z (as the dense kernels)
    T s;
#pragma unroll
    for (int d = 0; d < 6; ++d) {
        int32_t k = conn[(int64_t)d * n + j];
        T v = k >= 0 ? x[k] : outside;
        s = d == 0 ? v : s + v;
    }
    return s;
}

// NSB segments per block: thread t handles cell t of each of them, so every
// thread has NSB independent loads per operand in flight; each segment keeps
// its own canonical reduction (butterfly per warp, then the 8 warps).
#ifndef NB_SP_NSB
#define NB_SP_NSB 4
#endif
constexpr int NSB = NB_SP_NSB;
#ifndef NB_SP_MINB
#define NB_SP_MINB 0
#endif
#if NB_SP_MINB > 0
#define NB_SP_LB __launch_bounds__(SEG, NB_SP_MINB)
#else
#define NB_SP_LB __launch_bounds__(SEG)
#endif

template <int K>
__global__ void NB_SP_LB k_sp(SpArgs A) {
    __shared__ double sw[NSB][SEG / 32];
#if NB_SP_EARLY_STATUS
    if (K >= SPK_CG_MAP && K <= SPK_CG_R && A.sc->status != 0) return;
#endif
    const int t = threadIdx.x;
    // the segment-table entries do not depend on the solver status: load
    // them first so the status load and the table loads overlap (one
    // dependent hop fewer before the connectivity / operand loads)
    int e[NSB];
#pragma unroll
    for (int k = 0; k < NSB; ++k) {
        const int64_t q = (int64_t)blockIdx.x * NSB + k;
        e[k] = q < A.nseg ? __ldg(A.seg + A.seg0 + q) : -1;  // non-empty segment: plane << 16 | index
    }
#if !NB_SP_EARLY_STATUS
    if (K >= SPK_CG_MAP && K <= SPK_CG_R && A.sc->status != 0) return;
#endif
    int zl[NSB], sg[NSB];
    int64_t i[NSB], jj[NSB];
    bool valid[NSB];
#pragma unroll
    for (int k = 0; k < NSB; ++k) {
        zl[k] = -1;
        sg[k] = 0;
        valid[k] = false;
        jj[k] = 0;
        if (e[k] >= 0) {
            zl[k] = e[k] >> 16;
            sg[k] = e[k] & 0xffff;
            jj[k] = __ldg(A.pstart + zl[k]) + (int64_t)sg[k] * SEG + t;
            valid[k] = jj[k] < __ldg(A.pstart + zl[k] + 1);
        }
        i[k] = A.hl + jj[k];  // buffer index of own cell
    }
    double prod[NSB];
    if (K == SPK_DOT) {
        double a[NSB], b[NSB];
#pragma unroll
        for (int k = 0; k < NSB; ++k) {
            a[k] = valid[k] ? A.a[i[k]] : 0.0;
            b[k] = valid[k] ? A.b[i[k]] : 0.0;
        }
#pragma unroll
        for (int k = 0; k < NSB; ++k) prod[k] = __dmul_rn(a[k], b[k]);
    } else if (K == SPK_CG_INIT || K == SPK_CG_Q) {  // CG_INIT: r = b - A x; CG_Q: q = A p, <p, q>
        // all connectivity loads of the NSB cells first, then all gathers:
        // one table + one gather latency per thread instead of NSB of each
        const double outv = K == SPK_CG_INIT ? A.outside : 0.0;
        int32_t nbr[NSB][6];
#pragma unroll
        for (int k = 0; k < NSB; ++k)
#pragma unroll
            for (int d = 0; d < 6; ++d) nbr[k][d] = valid[k] ? __ldg(A.conn + (int64_t)d * A.n + jj[k]) : -1;
        double s[NSB], c[NSB], bb[NSB], v[NSB][6];
#pragma unroll
        for (int k = 0; k < NSB; ++k) {
            c[k] = valid[k] ? __ldg(A.a + i[k]) : 0.0;
            bb[k] = (K == SPK_CG_INIT && valid[k]) ? __ldg(A.b + i[k]) : 0.0;
        }
#pragma unroll
        for (int k = 0; k < NSB; ++k)
#pragma unroll
            for (int d = 0; d < 6; ++d) v[k][d] = nbr[k][d] >= 0 ? __ldg(A.a + nbr[k][d]) : outv;
#pragma unroll
        for (int k = 0; k < NSB; ++k) {  // canonical order -x, +x, -y, +y, -z, +z (sp_nsum)
            double t = v[k][0];
#pragma unroll
            for (int d = 1; d < 6; ++d) t = t + v[k][d];
            s[k] = valid[k] ? t : 0.0;
        }
#pragma unroll
        for (int k = 0; k < NSB; ++k) {
            prod[k] = 0.0;
            if (!valid[k]) continue;
            const double ac = fma(6.0, c[k], -s[k]);
            if (K == SPK_CG_INIT) {
                const double r = __dsub_rn(bb[k], ac);
                A.c[i[k]] = r;
                prod[k] = __dmul_rn(r, r);
            } else {
                A.c[i[k]] = ac;
                prod[k] = __dmul_rn(c[k], ac);
            }
        }
    } else if (K == SPK_CG_MAP) {  // x += alpha_prev p_old (pending); p = r + beta p_old
        const int pending = A.sc->pending;
        const double beta = A.sc->beta, ap = A.sc->alpha_prev;
        double po[NSB], rr[NSB], xx[NSB];
#pragma unroll
        for (int k = 0; k < NSB; ++k) {
            po[k] = valid[k] ? A.c[i[k]] : 0.0;
            rr[k] = valid[k] ? A.a[i[k]] : 0.0;
            xx[k] = (valid[k] && pending) ? A.d[i[k]] : 0.0;
        }
#pragma unroll
        for (int k = 0; k < NSB; ++k) {
            prod[k] = 0.0;
            if (!valid[k]) continue;
            if (pending) A.d[i[k]] = fma(ap, po[k], xx[k]);
            A.c[i[k]] = fma(beta, po[k], rr[k]);
        }
    } else {  // SPK_CG_R: r -= alpha q, <r, r>
        const double alpha = A.sc->alpha;
        double qq[NSB], rr[NSB];
#pragma unroll
        for (int k = 0; k < NSB; ++k) {
            qq[k] = valid[k] ? A.a[i[k]] : 0.0;
            rr[k] = valid[k] ? A.c[i[k]] : 0.0;
        }
#pragma unroll
        for (int k = 0; k < NSB; ++k) {
            prod[k] = 0.0;
            if (!valid[k]) continue;
            const double r = fma(-alpha, qq[k], rr[k]);
            A.c[i[k]] = r;
            prod[k] = __dmul_rn(r, r);
        }
    }
    if (K == SPK_DOT || K == SPK_CG_INIT || K == SPK_CG_Q || K == SPK_CG_R) {
        const int w = t >> 5;
#pragma unroll
        for (int k = 0; k < NSB; ++k) {
            const double v = warp_sum_canon(prod[k]);
            if ((t & 31) == 0) sw[k][w] = v;
        }
        __syncthreads();
        if (t < NSB && zl[t] >= 0) {
            double s = sw[t][0];
#pragma unroll
            for (int ww = 1; ww < SEG / 32; ++ww) s = __dadd_rn(s, sw[t][ww]);
            A.tp[(int64_t)(A.plane0 + zl[t]) * A.T + sg[t]] = s;
        }
    }
}

template <typename T>
__global__ void __launch_bounds__(SEG) k_sp_lap(const T *x, T *y, const int32_t *seg, int64_t seg0, const int64_t *pstart,
                                                const int32_t *conn, int64_t n, int64_t hl, T outside) {
    const int e = seg[seg0 + blockIdx.x];
    const int zl = e >> 16;
    const int64_t j = pstart[zl] + (int64_t)(e & 0xffff) * SEG + threadIdx.x;
    if (j >= pstart[zl + 1]) return;
    T s = sp_nsum(x, conn, n, j, outside);
    y[hl + j] = fma(T(-6), x[hl + j], s);
}

struct SpRun;
static bool sp_use_runs(const NbSparsePart &sp);
template <int K>
static nb_status sp_launch_runs(nb_grid *g, int p, const int32_t *list, const int32_t *gidx, int64_t s0, int64_t n,
                                SpArgs A, int plane_base, const char *name);

// launch over the non-empty segments of local planes [zb, ze)
template <int K>
static nb_status sp_launch(nb_grid *g, int p, int zb, int ze, SpArgs A, int plane_base, const char *name) {
    if (ze <= zb) return NB_OK;
    const NbSparsePart &sp = g->sp[p];
    const int64_t s0 = sp.seg_start[zb], s1 = sp.seg_start[ze];
    if (s1 <= s0) return NB_OK;
    if constexpr (K == SPK_CG_Q || K == SPK_CG_INIT)
        if (sp_use_runs(sp)) return sp_launch_runs<K>(g, p, sp.d_seg, nullptr, s0, s1 - s0, A, plane_base, name);
    A.seg = sp.d_seg;
    A.seg0 = s0;
    A.nseg = s1 - s0;
    A.pstart = sp.d_pstart;
    A.conn = sp.conn;
    A.n = sp.n;
    A.hl = sp.hl;
    A.plane0 = plane_base + g->parts[p].z0;
    A.T = g->T;
    A.tp = g->tp;
    LaunchScope ls(g, g->cs, name);
    k_sp<K><<<(unsigned)((s1 - s0 + NSB - 1) / NSB), SEG, 0, g->cs>>>(A);
    return nb_launch_check(name);
}

// launch over an explicit list of segment entries (plane << 16 | index)
template <int K>
static nb_status sp_launch_list(nb_grid *g, int p, const int32_t *list, int64_t n, SpArgs A, int plane_base,
                                const char *name) {
    if (n <= 0) return NB_OK;
    const NbSparsePart &sp = g->sp[p];
    if constexpr (K == SPK_CG_Q || K == SPK_CG_INIT)
        if (sp_use_runs(sp)) return sp_launch_runs<K>(g, p, list, sp.d_seg_bnd_gi, 0, n, A, plane_base, name);
    A.seg = list;
    A.seg0 = 0;
    A.nseg = n;
    A.pstart = sp.d_pstart;
    A.conn = sp.conn;
    A.n = sp.n;
    A.hl = sp.hl;
    A.plane0 = plane_base + g->parts[p].z0;
    A.T = g->T;
    A.tp = g->tp;
    LaunchScope ls(g, g->cs, name);
    k_sp<K><<<(unsigned)((n + NSB - 1) / NSB), SEG, 0, g->cs>>>(A);
    return nb_launch_check(name);
}

// the segments of partition p's boundary planes (those facing a neighbour);
// built at grid creation (never under graph capture)
static nb_status sp_bnd_segments(nb_grid *g, int p) {
    NbSparsePart &sp = g->sp[p];
    if (sp.n_seg_bnd >= 0) return NB_OK;
    const NbPart &q = g->parts[p];
    std::vector<int32_t> segs;
    auto add = [&](int zl) {
        for (int64_t k = 0; k < sp.seg_start[zl + 1] - sp.seg_start[zl]; ++k) segs.push_back((zl << 16) | (int)k);
    };
    if (q.lo >= 0) add(0);
    if (q.hi >= 0 && q.nz() > 1) add(q.nz() - 1);
    std::vector<int32_t> gi;  // index of each entry in the full (plane-major) segment table
    for (int32_t e : segs) gi.push_back((int32_t)(sp.seg_start[e >> 16] + (e & 0xffff)));
    NB_CUDA(cudaMalloc(&sp.d_seg_bnd, sizeof(int32_t) * std::max<size_t>(segs.size(), 1)));
    NB_CUDA(cudaMalloc(&sp.d_seg_bnd_gi, sizeof(int32_t) * std::max<size_t>(segs.size(), 1)));
    if (!segs.empty()) {
        NB_CUDA(cudaMemcpy(sp.d_seg_bnd, segs.data(), sizeof(int32_t) * segs.size(), cudaMemcpyHostToDevice));
        NB_CUDA(cudaMemcpy(sp.d_seg_bnd_gi, gi.data(), sizeof(int32_t) * gi.size(), cudaMemcpyHostToDevice));
    }
    sp.n_seg_bnd = (int64_t)segs.size();
    return NB_OK;
}

// ---------------------------------------------------------------------------
// x-runs (the C4 q pass without a per-cell connectivity table).  PAPER.md
// L248 stores the sparse grid "with their connectivity table" and leaves the
// format open; the 7-point stencil only needs, per run of consecutive active
// cells along x, whether the +-x ends continue and where the +-y / +-z
// neighbour run starts.  A run is cut wherever a neighbour row starts or
// stops being active, and at every 256-cell dot segment boundary, so each
// of the four offsets is constant over the run (or the whole run's neighbour
// is inactive -> outside).  24 B per run instead of 24 B per cell.
// ---------------------------------------------------------------------------
struct SpRun {
    int32_t start;   // own index of the first cell
    int16_t len;     // cells (<= SEG)
    int16_t flags;   // bit 0: the first cell's -x neighbour is active (= own cell start - 1), bit 1: the last cell's +x
    int32_t off[4];  // -y, +y, -z, +z: buffer index of the neighbour minus the cell's own buffer index
};
constexpr int32_t SP_NONE = INT32_MIN;
static_assert(sizeof(SpRun) == 24, "SpRun layout");

static nb_status sp_build_runs(nb_grid *g, int p) {
    NbSparsePart &sp = g->sp[p];
    const NbPart &q = g->parts[p];
    const int nx = g->nx, ny = g->ny;
    const int64_t plane = (int64_t)nx * ny;
    struct XRun {
        int x0, x1;
        int64_t rank;  // rank of the cell x0 among its plane's active cells
    };
    // planes z0 - 1 .. z1 (halo planes only where a neighbour partition exists)
    const int zlo = q.lo >= 0 ? q.z0 - 1 : q.z0, zhi = q.hi >= 0 ? q.z1 + 1 : q.z1;
    std::vector<std::vector<XRun>> runs(zhi - zlo);
    std::vector<std::vector<int32_t>> rowbeg(zhi - zlo);
    for (int z = zlo; z < zhi; ++z) {
        auto &R = runs[z - zlo];
        auto &B = rowbeg[z - zlo];
        B.assign(ny + 1, 0);
        const uint8_t *m = g->host_mask.data() + (int64_t)z * plane;
        int64_t rank = 0;
        for (int y = 0; y < ny; ++y) {
            B[y] = (int32_t)R.size();
            const uint8_t *row = m + (int64_t)y * nx;
            for (int x = 0; x < nx;) {
                if (!row[x]) {
                    ++x;
                    continue;
                }
                int x0 = x;
                while (x < nx && row[x]) ++x;
                R.push_back({x0, x, rank});
                rank += x - x0;
            }
        }
        B[ny] = (int32_t)R.size();
    }
    // buffer index of the first cell of plane z ([halo_lo | own | halo_hi])
    auto base = [&](int z) -> int64_t {
        if (z < q.z0) return 0;
        if (z >= q.z1) return sp.hl + sp.n;
        return sp.hl + sp.pstart[z - q.z0];
    };
    std::vector<SpRun> out;
    std::vector<int32_t> rseg;  // first run of every segment, plane-major
    std::vector<int> cuts;
    for (int z = q.z0; z < q.z1; ++z) {
        const int zl = z - q.z0;
        const auto &R = runs[z - zlo];
        const auto &B = rowbeg[z - zlo];
        const int64_t p0 = sp.pstart[zl];
        for (int y = 0; y < ny; ++y) {
            // neighbour rows: -y, +y, -z, +z (plane index into runs, row) or none
            int nz_[4], ny_[4];
            nz_[0] = z, ny_[0] = y - 1;
            nz_[1] = z, ny_[1] = y + 1;
            nz_[2] = z - 1, ny_[2] = y;
            nz_[3] = z + 1, ny_[3] = y;
            bool has[4];
            for (int d = 0; d < 4; ++d) has[d] = ny_[d] >= 0 && ny_[d] < ny && nz_[d] >= zlo && nz_[d] < zhi;
            for (int k = B[y]; k < B[y + 1]; ++k) {
                const XRun &r = R[k];
                cuts.clear();
                cuts.push_back(r.x0);
                cuts.push_back(r.x1);
                for (int d = 0; d < 4; ++d) {
                    if (!has[d]) continue;
                    const auto &NR = runs[nz_[d] - zlo];
                    const auto &NB = rowbeg[nz_[d] - zlo];
                    for (int m = NB[ny_[d]]; m < NB[ny_[d] + 1]; ++m) {
                        if (NR[m].x0 > r.x0 && NR[m].x0 < r.x1) cuts.push_back(NR[m].x0);
                        if (NR[m].x1 > r.x0 && NR[m].x1 < r.x1) cuts.push_back(NR[m].x1);
                    }
                }
                // 256-cell segment boundaries of the plane's own order
                for (int64_t sj = (r.rank + SEG - 1) / SEG * SEG; sj < r.rank + (r.x1 - r.x0); sj += SEG)
                    if (sj > r.rank) cuts.push_back(r.x0 + (int)(sj - r.rank));
                std::sort(cuts.begin(), cuts.end());
                cuts.erase(std::unique(cuts.begin(), cuts.end()), cuts.end());
                for (size_t c = 0; c + 1 < cuts.size(); ++c) {
                    const int u = cuts[c], v = cuts[c + 1];
                    SpRun o;
                    const int64_t j = p0 + r.rank + (u - r.x0);
                    o.start = (int32_t)j;
                    o.len = (int16_t)(v - u);
                    o.flags = (int16_t)((u > r.x0 ? 1 : 0) | (v < r.x1 ? 2 : 0));
                    const int64_t own = sp.hl + j;
                    for (int d = 0; d < 4; ++d) {
                        o.off[d] = SP_NONE;
                        if (!has[d]) continue;
                        const auto &NR = runs[nz_[d] - zlo];
                        const auto &NB = rowbeg[nz_[d] - zlo];
                        for (int m = NB[ny_[d]]; m < NB[ny_[d] + 1]; ++m)
                            if (NR[m].x0 <= u && u < NR[m].x1) {
                                o.off[d] = (int32_t)(base(nz_[d]) + NR[m].rank + (u - NR[m].x0) - own);
                                break;
                            }
                    }
                    if ((j - p0) % SEG == 0) rseg.push_back((int32_t)out.size());
                    out.push_back(o);
                }
            }
        }
    }
    rseg.push_back((int32_t)out.size());
    if ((int64_t)rseg.size() != sp.seg_start.back() + 1)
        NB_FAIL(NB_ESTATE, "sparse x-runs: %zu segment starts, expected %lld", rseg.size() - 1,
                (long long)sp.seg_start.back());
    // the device table, segment-indexed so that a thread finds its cell's
    // entry from (segment, lane) alone: per cell {-z, +z, -y << 2 | x flags,
    // +y} (16 B; -y offsets fit 30 bits), per segment {first own cell,
    // cells, plane << 16 | index}
    const int64_t nseg = (int64_t)rseg.size() - 1;
    std::vector<int4> nbr((size_t)nseg * SEG, make_int4(SP_NONE, SP_NONE, (SP_NONE >> 2) * 4, SP_NONE));
    std::vector<int4> info((size_t)std::max<int64_t>(nseg, 1));
    int64_t sgi = 0;
    for (int zl = 0; zl < q.nz(); ++zl)
        for (int64_t k = 0; k < sp.seg_start[zl + 1] - sp.seg_start[zl]; ++k, ++sgi) {
            const int64_t j0 = sp.pstart[zl] + k * SEG;
            const int64_t cnt = std::min<int64_t>(SEG, sp.pstart[zl + 1] - j0);
            info[sgi] = make_int4((int32_t)j0, (int32_t)cnt, (zl << 16) | (int)k, 0);
            for (int32_t m = rseg[sgi]; m < rseg[sgi + 1]; ++m) {
                const SpRun &r = out[m];
                for (int c = 0; c < r.len; ++c) {
                    const int64_t j = r.start + c;
                    const int fx = ((c > 0 || (r.flags & 1)) ? 1 : 0) | ((c < r.len - 1 || (r.flags & 2)) ? 2 : 0);
                    const int32_t ylo = r.off[0] == SP_NONE ? (SP_NONE >> 2) : r.off[0];
                    if (ylo < -(1 << 29) || ylo >= (1 << 29))
                        NB_FAIL(NB_EUNSUPPORTED, "sparse neighbour table: -y offset out of range");
                    nbr[(size_t)sgi * SEG + (j - j0)] = make_int4(r.off[2], r.off[3], (int32_t)((uint32_t)ylo << 2) | fx,
                                                                  r.off[1]);
                }
            }
        }
    NB_CUDA(cudaMalloc(&sp.d_nbr, sizeof(int4) * std::max<size_t>(nbr.size(), 1)));
    NB_CUDA(cudaMalloc(&sp.d_seginfo, sizeof(int4) * info.size()));
    if (!nbr.empty()) NB_CUDA(cudaMemcpy(sp.d_nbr, nbr.data(), sizeof(int4) * nbr.size(), cudaMemcpyHostToDevice));
    NB_CUDA(cudaMemcpy(sp.d_seginfo, info.data(), sizeof(int4) * info.size(), cudaMemcpyHostToDevice));
    sp.n_runs = (int64_t)out.size();
    return NB_OK;
}

// 2 segments per block at 6 blocks per SM (40 registers): q pass 0.267 ms
// at 512^3 on the sphere, against 0.284 (2, 5), 0.299 (1, 6 or 8), 0.287
// (4, 3), 0.336 (2, 7: spills) and 0.317 for the connectivity-table path
#ifndef NB_SPR_MINB
#define NB_SPR_MINB 6
#endif
#ifndef NB_SPR_NSB
#define NB_SPR_NSB 2
#endif
constexpr int NSBR = NB_SPR_NSB;  // segments per block of the table-indexed passes
// The 7-point CG passes on the segment-indexed neighbour table
// (SPK_CG_Q: q = A p, <p, q>; SPK_CG_INIT: r = b - A x, <r, r>): the same
// cells per thread, the same canonical neighbour order -x, +x, -y, +y, -z,
// +z and the same per-segment dot tree as k_sp, so the results are bitwise
// those of the connectivity-table path.  The table is indexed by (segment,
// lane): ONE dependent level (segment info + the cell's 16-byte entry, both
// addressed from blockIdx / threadIdx) before the operand gathers, instead
// of segment entry -> plane start -> 24-byte connectivity -> gathers.
template <int K>
__global__ void __launch_bounds__(SEG, NB_SPR_MINB) k_sp_runs(SpArgs A, const int4 *__restrict__ nbrt,
                                                             const int4 *__restrict__ seginfo,
                                                             const int32_t *__restrict__ gidx) {
    __shared__ double sw[NSBR][SEG / 32];
    const int t = threadIdx.x;
    // L2 prefetch of the table entries and operand cells of the block A.pf
    // blocks ahead (blocks start in index order): when that block runs, its
    // table loads and its +z gathers hit L2 instead of DRAM, which takes one
    // DRAM latency off each cell's dependent chain.  The operand window is
    // estimated from the mean cells per segment (a prefetch only moves data).
    if (A.pf > 0 && gidx == nullptr && t < 2) {
        const int64_t qa = ((int64_t)blockIdx.x + A.pf) * NSBR;
        if (qa < A.nseg) {
            const int64_t nsa = A.nseg - qa < NSBR ? A.nseg - qa : NSBR;
            if (t == 0) {
                nb_prefetch_l2(nbrt + (A.seg0 + qa) * SEG, (uint32_t)(nsa * SEG * sizeof(int4)));
            } else {
                const int64_t c0 = A.hl + (int64_t)((float)(A.seg0 + qa) * A.cps);
                const int64_t a0 = (c0 - 64) & ~(int64_t)15;
                const int64_t lim = A.hl + A.n;
                if (a0 >= 0 && a0 + (NSBR * SEG + 128) <= lim)
                    nb_prefetch_l2(A.a + a0, (uint32_t)((NSBR * SEG + 128) * sizeof(double)));
            }
        }
    }
    int4 inf[NSBR], nb4[NSBR];
#pragma unroll
    for (int k = 0; k < NSBR; ++k) {
        const int64_t q = (int64_t)blockIdx.x * NSBR + k;
        const int64_t qc = q < A.nseg ? q : A.nseg - 1;
        const int64_t gi = gidx ? (int64_t)__ldg(gidx + qc) : A.seg0 + qc;
        inf[k] = __ldg(seginfo + gi);
        nb4[k] = __ldg(nbrt + gi * SEG + t);
        if (q >= A.nseg) inf[k].y = 0;  // no cells
    }
    if (K == SPK_CG_Q && A.sc->status != 0) return;
    const double outv = K == SPK_CG_INIT ? A.outside : 0.0;
    int64_t i[NSBR];
    bool valid[NSBR];
    int32_t nb[NSBR][6];
#pragma unroll
    for (int k = 0; k < NSBR; ++k) {
        valid[k] = t < inf[k].y;
        const int32_t ii = (int32_t)(A.hl + inf[k].x + t);
        i[k] = ii;
        const int fx = nb4[k].z & 3;
        const int32_t ylo = nb4[k].z >> 2;
        nb[k][0] = valid[k] && (fx & 1) ? ii - 1 : -1;
        nb[k][1] = valid[k] && (fx & 2) ? ii + 1 : -1;
        nb[k][2] = valid[k] && ylo != (SP_NONE >> 2) ? ii + ylo : -1;
        nb[k][3] = valid[k] && nb4[k].w != SP_NONE ? ii + nb4[k].w : -1;
        nb[k][4] = valid[k] && nb4[k].x != SP_NONE ? ii + nb4[k].x : -1;
        nb[k][5] = valid[k] && nb4[k].y != SP_NONE ? ii + nb4[k].y : -1;
    }
    double c[NSBR], bb[NSBR], v[NSBR][6];
#pragma unroll
    for (int k = 0; k < NSBR; ++k) {
        c[k] = valid[k] ? __ldg(A.a + i[k]) : 0.0;
        bb[k] = (K == SPK_CG_INIT && valid[k]) ? __ldg(A.b + i[k]) : 0.0;
    }
#pragma unroll
    for (int k = 0; k < NSBR; ++k)
#pragma unroll
        for (int d = 0; d < 6; ++d) v[k][d] = nb[k][d] >= 0 ? __ldg(A.a + nb[k][d]) : outv;
    double prod[NSBR];
#pragma unroll
    for (int k = 0; k < NSBR; ++k) {
        prod[k] = 0.0;
        if (!valid[k]) continue;
        double s = v[k][0];
#pragma unroll
        for (int d = 1; d < 6; ++d) s = s + v[k][d];
        const double ac = fma(6.0, c[k], -s);
        if (K == SPK_CG_INIT) {
            const double r = __dsub_rn(bb[k], ac);
            A.c[i[k]] = r;
            prod[k] = __dmul_rn(r, r);
        } else {
            A.c[i[k]] = ac;
            prod[k] = __dmul_rn(c[k], ac);
        }
    }
    const int w = t >> 5;
    warp_sums_store<NSBR>(prod, t & 31, &sw[0][w], SEG / 32);
    __syncthreads();
    if (t < NSBR) {
        int4 it = inf[0];
#pragma unroll
        for (int k = 1; k < NSBR; ++k)
            if (t == k) it = inf[k];
        if (it.y > 0) {
            double sum = sw[t][0];
#pragma unroll
            for (int ww = 1; ww < SEG / 32; ++ww) sum = __dadd_rn(sum, sw[t][ww]);
            A.tp[(int64_t)(A.plane0 + (it.z >> 16)) * A.T + (it.z & 0xffff)] = sum;
        }
    }
}

static bool sp_use_runs(const NbSparsePart &sp) { return sp.d_nbr && !getenv("NB_SP_CONN"); }

template <int K>
static nb_status sp_launch_runs(nb_grid *g, int p, const int32_t *list, const int32_t *gidx, int64_t s0, int64_t n,
                                SpArgs A, int plane_base, const char *name) {
    const NbSparsePart &sp = g->sp[p];
    A.seg = list;
    A.seg0 = s0;
    A.nseg = n;
    A.pstart = sp.d_pstart;
    A.n = sp.n;
    A.hl = sp.hl;
    A.plane0 = plane_base + g->parts[p].z0;
    A.T = g->T;
    A.tp = g->tp;
    {
        // 300-1500 blocks ahead measured equal (0.242 ms vs 0.269 without at
        // 512^3); 3000 loses the lines before use.  NB_SPR_PF=0 disables.
        static const int pf = getenv("NB_SPR_PF") ? atoi(getenv("NB_SPR_PF")) : 600;
        A.pf = gidx ? 0 : pf;
        A.cps = sp.seg_start.back() > 0 ? (float)((double)sp.n / (double)sp.seg_start.back()) : 256.f;
    }
    LaunchScope ls(g, g->cs, name);
    k_sp_runs<K><<<(unsigned)((n + NSBR - 1) / NSBR), SEG, 0, g->cs>>>(A, (const int4 *)sp.d_nbr,
                                                                    (const int4 *)sp.d_seginfo, gidx);
    return nb_launch_check(name);
}

nb_status nb_sparse_dot_partials(const nb_field *x, const nb_field *y) {
    nb_grid *g = x->g;
    if (x->dt != NB_F64) NB_FAIL(NB_EUNSUPPORTED, "sparse dot: fp64 fields");
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbSparsePart &sp = g->sp[p];
        for (int c = 0; c < x->card; ++c) {
            SpArgs A{};
            A.a = (const double *)x->base[p] + (int64_t)c * sp.cs;
            A.b = (const double *)y->base[p] + (int64_t)c * sp.cs;
            NB_TRY(sp_launch<SPK_DOT>(g, p, 0, g->parts[p].nz(), A, c * g->nz, "k_sp_dot"));
        }
    }
    return NB_OK;
}

nb_status nb_sparse_laplace7(const nb_field *x, nb_field *y, nb_view v) {
    nb_grid *g = x->g;
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbSparsePart &sp = g->sp[p];
        for (auto rg : view_ranges(g, p, v)) {
            const int64_t s0 = sp.seg_start[rg.first], s1 = sp.seg_start[rg.second];
            if (s1 <= s0) continue;
            LaunchScope ls(g, g->cs, "k_sp_lap");
            if (x->dt == NB_F64)
                k_sp_lap<double><<<(unsigned)(s1 - s0), SEG, 0, g->cs>>>((const double *)x->base[p], (double *)y->base[p],
                                                                         sp.d_seg, s0, sp.d_pstart, sp.conn, sp.n,
                                                                         sp.hl, x->outside);
            else
                k_sp_lap<float><<<(unsigned)(s1 - s0), SEG, 0, g->cs>>>((const float *)x->base[p], (float *)y->base[p],
                                                                        sp.d_seg, s0, sp.d_pstart, sp.conn, sp.n, sp.hl,
                                                                        (float)x->outside);
            NB_TRY(nb_launch_check("k_sp_lap"));
        }
    }
    return NB_OK;
}

// ---------------------------------------------------------------------------
// sparse CG: three passes per iteration (104 B per active cell incl. the
// 24 B connectivity): map (x deferred update, p = r + beta p) -> halo(p) ->
// q = A p, <p,q> -> alpha -> r -= alpha q, <r,r> -> beta
// ---------------------------------------------------------------------------
static nb_status sp_cg_box_init(nb_cg *cg);
bool nb_sparse_cg_boxed();

nb_status nb_sparse_cg_init(nb_cg *cg) {
    nb_grid *g = cg->g;
    if (nb_sparse_cg_boxed() && cg->prm.op == NB_OP_LAPLACE7) {
        cg->sp_box = cg->pingpong = true;
        return sp_cg_box_init(cg);
    }
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        SpArgs A{};
        A.a = (const double *)cg->x->base[p];
        A.b = (const double *)cg->b->base[p];
        A.c = (double *)cg->r->base[p];
        A.outside = cg->x->outside;
        NB_TRY(sp_launch<SPK_CG_INIT>(g, p, 0, g->parts[p].nz(), A, 0, "k_sp_cg_init"));
    }
    return nb_reduce_finalize(g, 1, FIN_CG_INIT, cg->sc, 0);
}

// OCC with occ != NONE and a transfer that actually
// runs asynchronously (the peer or NCCL transport across processes, or
// NB_HALO_STREAM): the map of the boundary planes (the neighbours' halos)
// first, the halo transfer of p started on the halo stream, the interior map
// and interior q pass enqueued while it is in flight, then the wait and the
// q pass of the boundary planes (both planes in one launch).  Every cell runs
// the same arithmetic and the dot partials are per plane, so all schedules
// give the same bits.  Extended / Two-way split the map as well (the reduce
// is per plane in any case); Standard maps every plane before the transfer.
// In one process with fused halos the copies are stream-ordered work with
// nothing to overlap, and the serial schedule runs.
static nb_status sp_cg_box_iter(nb_cg *cg, int parity);

nb_status nb_sparse_cg_hooks(nb_cg *cg, int parity) {
    if (cg->sp_box) return sp_cg_box_iter(cg, parity);
    nb_grid *g = cg->g;
    nb_field *p_ = cg->p[0];
    const nb_occ occ = cg->prm.occ;
    const bool split = occ != NB_OCC_NONE && g->nparts > 1 && (nb_is_peer(g) || nb_halo_on_stream(g));
    const bool split_map = split && occ != NB_OCC_STANDARD;
    auto map_args = [&](int p) {
        SpArgs A{};
        A.a = (const double *)cg->r->base[p];
        A.c = (double *)p_->base[p];
        A.d = (double *)cg->x->base[p];
        A.sc = cg->sc;
        return A;
    };
    auto q_args = [&](int p) {
        SpArgs A{};
        A.a = (const double *)p_->base[p];
        A.c = (double *)cg->q->base[p];
        A.sc = cg->sc;
        return A;
    };
    // interior planes [ib, ie) of a partition: those whose neighbours are own planes
    auto inner = [&](int p, int *ib, int *ie) {
        const NbPart &q = g->parts[p];
        *ib = q.lo >= 0 ? 1 : 0;
        *ie = q.nz() - (q.hi >= 0 ? 1 : 0);
        if (*ie < *ib) *ie = *ib;
    };
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        if (split_map) {
            const NbSparsePart &sp = g->sp[p];
            NB_TRY(sp_launch_list<SPK_CG_MAP>(g, p, sp.d_seg_bnd, sp.n_seg_bnd, map_args(p), 0, "k_sp_cg_map"));
        } else {
            NB_TRY(sp_launch<SPK_CG_MAP>(g, p, 0, g->parts[p].nz(), map_args(p), 0, "k_sp_cg_map"));
        }
    }
    if (!split) {
        NB_TRY(nb_sparse_halo_update(p_));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p)
            NB_TRY(sp_launch<SPK_CG_Q>(g, p, 0, g->parts[p].nz(), q_args(p), 0, "k_sp_cg_q"));
    } else {
        NB_TRY(nb_halo_split_begin(p_, 0, 1, cg->hs));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            int ib, ie;
            inner(p, &ib, &ie);
            if (split_map) NB_TRY(sp_launch<SPK_CG_MAP>(g, p, ib, ie, map_args(p), 0, "k_sp_cg_map"));
            NB_TRY(sp_launch<SPK_CG_Q>(g, p, ib, ie, q_args(p), 0, "k_sp_cg_q"));
        }
        NB_TRY(nb_halo_split_wait(g, cg->hs));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            const NbSparsePart &sp = g->sp[p];
            NB_TRY(sp_launch_list<SPK_CG_Q>(g, p, sp.d_seg_bnd, sp.n_seg_bnd, q_args(p), 0, "k_sp_cg_q"));
        }
    }
    NB_TRY(nb_reduce_finalize(g, 1, FIN_CG_PQ, cg->sc, 0));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        SpArgs A{};
        A.a = (const double *)cg->q->base[p];
        A.c = (double *)cg->r->base[p];
        A.sc = cg->sc;
        NB_TRY(sp_launch<SPK_CG_R>(g, p, 0, g->parts[p].nz(), A, 0, "k_sp_cg_r"));
    }
    NB_TRY(nb_reduce_finalize(g, 1, FIN_CG_RR, cg->sc, 0));
    cg->k += 1;
    return NB_OK;
}

// ===========================================================================
// The 2-phase CG of the dense grid (64 B per cell, Ap
// recomputed, not stored) on the element-sparse grid (a9).  A CTA owns a
// 32 x 8 tile of the bounding box for a z-chunk and stages, per plane, the
// 34 x 10 box around it from the compact arrays (8-byte cp.async, zero-fill
// = the outside value 0 for inactive cells; buffer index = row word index +
// popcount, the FEM box tables), three planes read while six more are in
// flight (NB_SPB_NST = 9 slots: a 7-point plane is little work, so the
// prefetch must be deep to keep ~50 KB per SM in flight).
//   phase A (PH 0): own planes stage r and p_old; each thread turns its own
//     box cells into p_new = r + beta p_old (fma(beta, p_old, r), the map's
//     arithmetic) right after its copies land; halo planes stage the
//     exchanged p_new.  Every active node stores p_new and, pending, x +=
//     alpha_prev p_old; q = A p_new (canonical 7-point order) feeds <p_new, q>.
//   phase B (PH 1): stages p_new, recomputes A p_new, r = fma(-alpha, A p, r),
//     <r, r>.
//   set-up (PH 2): stages x, r = b - A x, <r, r>.
// 40 + 24 B per active cell and iteration (+ the ring rows from L2) against
// the 96 B of the map / q / r schedule.  The dots are per 32 x 8 tile of a
// plane in the dense canonical order (warp = tile row, rows added in y,
// tiles by the finalize tree over the plane's tiles): every tile of every
// chunk is launched (empty ones write zero partials), into the grid's sp_tp.
// ===========================================================================
#ifndef NB_SPB_NST
#define NB_SPB_NST 9  // ring slots: planes pl-2 .. pl read, pl+1 .. pl+6 in flight (1 component: 2.7 KB a slot)
#endif
#ifndef NB_SPB_ZC
#define NB_SPB_ZC 32
#endif
#ifndef NB_SPB_MINB
#define NB_SPB_MINB 4  // 64 registers: 1.42 against 1.56 ms per iteration at 3
#endif
#define SPB_NST NB_SPB_NST
#define SPB_ZC NB_SPB_ZC
#define SPB_W 34
#define SPB_H 10
#define SPB_C (SPB_W * SPB_H)

struct SpCgBoxArgs {
    const int4 *items;  // {tile x (| 1 << 30: no active cell), tile y, zs, ze}
    const uint32_t *rm;
    const int32_t *ri;
    int rw, nx, ny, gz0, nzl, NZ, T, tx;
    double *tp;
    const double *u;      // PH 0: halo planes' p_new (the p_new buffer); PH 1: p_new; PH 2: x
    const double *r, *po;  // PH 0: r, p_old (own planes)
    const double *b;       // PH 2
    double *pn, *x;        // PH 0
    double *ro;            // PH 1 / 2: r (read-modify-write / written)
    const CgScal *sc;
};

__device__ __forceinline__ void spb_cp8(double *dst, const double *src, bool on) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(d), "l"(src), "r"(on ? 8 : 0) : "memory");
}

template <int PH>
struct SpbCfg {
    static constexpr int NPO = PH == 0 ? SPB_NST - 1 : 0;  // p_old slots (planes pl-1 .. pl+AHEAD)
    static constexpr int SMEM = (SPB_NST + NPO) * SPB_C * 8;
};

template <int PH>
__global__ void __launch_bounds__(256, NB_SPB_MINB) k_sp_cg_box(SpCgBoxArgs A) {
    extern __shared__ __align__(16) double spb_sm[];
    double(*S)[SPB_C] = reinterpret_cast<double(*)[SPB_C]>(spb_sm);
    double(*PO)[SPB_C] = reinterpret_cast<double(*)[SPB_C]>(spb_sm + SPB_NST * SPB_C);
    constexpr int NPO = SpbCfg<PH>::NPO;
    __shared__ uint64_t RB[SPB_NST][SPB_H];
    __shared__ double sw[2][8];
    if (PH != 2 && A.sc->status != 0) return;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const int4 it = A.items[blockIdx.x];
    const int bxi = it.x & 0x3fffffff, x0 = bxi * 32, y0 = it.y * 8, zs = it.z, ze = it.w;
    const int nout = ze - zs, np = nout + 2;
    const int tile = it.y * A.tx + bxi;
    if (it.x & 0x40000000) {  // no active cell in the tile's chunk: zero partials
        for (int o = tid; o < nout; o += 256) A.tp[(int64_t)(A.gz0 + zs + o) * A.T + tile] = 0.0;
        return;
    }
    const int wx = bxi;
    double beta = 0.0, ap = 0.0, alpha = 0.0;
    bool dox = false;
    if constexpr (PH == 0) {
        beta = A.sc->beta;
        ap = A.sc->alpha_prev;
        dox = A.sc->pending != 0;
    }
    if constexpr (PH == 1) alpha = A.sc->alpha;
    int cx[2], cy[2];
    bool cv[2];
#pragma unroll
    for (int k = 0; k < 2; ++k) {
        const int e = tid + 256 * k;
        cx[k] = x0 - 1 + e % SPB_W;
        cy[k] = y0 - 1 + e / SPB_W;
        cv[k] = e < SPB_C && cx[k] >= 0 && cx[k] < A.nx && cy[k] >= 0 && cy[k] < A.ny;
    }
    const int rt = tid - (SPB_C - 256);  // box row built by a one-cell thread
    const int ry = y0 - 1 + rt;
    const bool rown = rt >= 0 && rt < SPB_H;
    const bool rv = rown && ry >= 0 && ry < A.ny;
    uint32_t tm[2] = {0u, 0u}, rl = 0u, rmid = 0u, rh = 0u;
    int32_t ti[2] = {0, 0};
    auto own = [&](int pl) { const int zl = zs - 1 + pl; return zl >= 0 && zl < A.nzl; };
    auto fetch = [&](int pl) {
        const int64_t row0 = (int64_t)(zs + pl) * A.ny;
#pragma unroll
        for (int k = 0; k < 2; ++k)
            if (cv[k]) {
                const int64_t q = (row0 + cy[k]) * A.rw + (cx[k] >> 5);
                tm[k] = __ldg(A.rm + q);
                ti[k] = __ldg(A.ri + q);
            }
        if (rv) {
            const uint32_t *r = A.rm + (row0 + ry) * A.rw;
            rl = wx > 0 ? __ldg(r + wx - 1) : 0u;
            rmid = __ldg(r + wx);
            rh = wx + 1 < A.rw ? __ldg(r + wx + 1) : 0u;
        }
    };
    auto issue = [&](int pl) {
        const int st = pl % SPB_NST;
        const bool form = PH == 0 && own(pl);
#pragma unroll
        for (int k = 0; k < 2; ++k) {
            const int e = tid + 256 * k;
            if (e < SPB_C) {
                const unsigned b = (unsigned)cx[k] & 31u;
                const bool act = cv[k] && ((tm[k] >> b) & 1u);
                const int64_t idx = act ? ti[k] + __popc(tm[k] & ((1u << b) - 1u)) : 0;
                if (form) {
                    spb_cp8(&S[st][e], A.r + idx, act);
                    spb_cp8(&PO[pl % (NPO ? NPO : 1)][e], A.po + idx, act);
                } else {
                    spb_cp8(&S[st][e], A.u + idx, act);
                }
            }
        }
        if (rown)
            RB[st][rt] = rv ? (uint64_t)(rl >> 31) | ((uint64_t)rmid << 1) | ((uint64_t)(rh & 1u) << 33) : 0ull;
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    constexpr int AHEAD = SPB_NST - 3;
#pragma unroll 1
    for (int pl = 0; pl < AHEAD; ++pl) {
        if (pl < np) {
            fetch(pl);
            issue(pl);
        } else {
            asm volatile("cp.async.commit_group;" ::: "memory");
        }
    }
    if (AHEAD < np) fetch(AHEAD);
    const int x = x0 + lane, y = y0 + w;
    const bool in = x < A.nx && y < A.ny;
    const int ce = (w + 1) * SPB_W + lane + 1;
    const uint32_t lmask = (1u << lane) - 1u;
    double vo = 0.0, bo = 0.0;  // x (PH 0) or r (PH 1) or b (PH 2) of the next output, a step ahead
    int32_t oi = 0;
    int64_t ic = 0;
#pragma unroll 1
    for (int pl = 0; pl < np; ++pl) {
        asm volatile("cp.async.wait_group %0;" ::"n"(AHEAD - 1) : "memory");
        const int sl = pl % SPB_NST;
        if constexpr (PH == 0) {
            if (own(pl)) {
#pragma unroll
                for (int k = 0; k < 2; ++k) {
                    const int e = tid + 256 * k;
                    if (e < SPB_C) S[sl][e] = fma(beta, PO[pl % NPO][e], S[sl][e]);
                }
            }
        }
        __syncthreads();  // plane pl landed (p_new formed); slot of plane pl-3 free; sw of output pl-3 written
        if (pl >= 3 && tid == 0) {  // tile partial of output pl-3: rows in increasing y
            const double(&v)[8] = sw[(pl - 3) & 1];
            double s = v[0];
#pragma unroll
            for (int k = 1; k < 8; ++k) s = __dadd_rn(s, v[k]);
            A.tp[(int64_t)(A.gz0 + zs + pl - 3) * A.T + tile] = s;
        }
        if (pl + AHEAD < np) issue(pl + AHEAD);
        else asm volatile("cp.async.commit_group;" ::: "memory");
        if (pl + AHEAD + 1 < np) fetch(pl + AHEAD + 1);
        if (pl >= 2) {  // output pl-2: centre plane pl-1
            const int s0 = (pl + SPB_NST - 2) % SPB_NST, s1 = (pl + SPB_NST - 1) % SPB_NST;
            double prod = 0.0;
            if (in && ((RB[s1][w + 1] >> (lane + 1)) & 1u)) {
                const double c = S[s1][ce];
                double sum = S[s1][ce - 1];
                sum = sum + S[s1][ce + 1];
                sum = sum + S[s1][ce - SPB_W];
                sum = sum + S[s1][ce + SPB_W];
                sum = sum + S[s0][ce];
                sum = sum + S[sl][ce];
                const double ac = fma(6.0, c, -sum);
                if constexpr (PH == 0) {
                    __stcs(A.pn + ic, c);
                    if (dox) __stcs(A.x + ic, fma(ap, PO[(pl - 1) % NPO][ce], vo));
                    prod = __dmul_rn(c, ac);
                } else if constexpr (PH == 1) {
                    const double r = fma(-alpha, ac, vo);
                    __stcs(A.ro + ic, r);
                    prod = __dmul_rn(r, r);
                } else {
                    const double r = __dsub_rn(bo, ac);
                    A.ro[ic] = r;
                    prod = __dmul_rn(r, r);
                }
            }
            const double ws = warp_sum_canon(prod);
            if (lane == 0) sw[(pl - 2) & 1][w] = ws;
        }
        // the next output (pl - 1, centre plane pl): buffer index, operand a step ahead
        if (pl >= 1 && pl - 1 < nout) {
            const uint64_t cb = RB[sl][w + 1];
            ic = oi + __popc((uint32_t)(cb >> 1) & lmask);
            if (in && ((cb >> (lane + 1)) & 1u)) {
                if constexpr (PH == 0) {
                    if (dox) vo = __ldcs(A.x + ic);
                } else if constexpr (PH == 1) {
                    vo = __ldcs(A.ro + ic);
                } else {
                    bo = __ldg(A.b + ic);
                }
            }
        }
        if (in && pl < nout) oi = __ldg(A.ri + ((int64_t)(zs + pl + 1) * A.ny + y) * A.rw + wx);
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncthreads();
    if (tid == 0) {  // the last output's tile partial
        const double(&v)[8] = sw[(nout - 1) & 1];
        double s = v[0];
#pragma unroll
        for (int k = 1; k < 8; ++k) s = __dadd_rn(s, v[k]);
        A.tp[(int64_t)(A.gz0 + zs + nout - 1) * A.T + tile] = s;
    }
}

// work items of the box CG: EVERY (tile, chunk) of the plane ranges (the
// tile partials of every tile are rewritten), empty ones flagged; cached
static nb_status spb_items(nb_grid *g, int p, const std::vector<int> &ranges, const int4 **items, int64_t *n) {
    NB_TRY(nb_sparse_fem_box_tables(g));
    NbSparsePart &sp = g->sp[p];
    std::vector<int> key = ranges;
    key.push_back(-SPB_ZC);  // distinct from the FEM operator's lists
    auto it = sp.box_lists.find(key);
    if (it == sp.box_lists.end()) {
        const int tx = (g->nx + 31) / 32, ty = (g->ny + 7) / 8;
        std::vector<int4> v;
        for (size_t r = 0; r + 1 < ranges.size(); r += 2)
            for (int zs = ranges[r]; zs < ranges[r + 1]; zs += SPB_ZC) {
                const int ze = std::min(zs + SPB_ZC, ranges[r + 1]);
                for (int by = 0; by < ty; ++by)
                    for (int bx = 0; bx < tx; ++bx) {
                        bool any = false;
                        for (int zl = zs; zl < ze && !any; ++zl)
                            any = sp.tile_any[((size_t)zl * ty + by) * tx + bx] != 0;
                        v.push_back(make_int4(bx | (any ? 0 : 0x40000000), by, zs, ze));
                    }
            }
        int4 *d = nullptr;
        if (!v.empty()) {
            DeviceGuard dg(g->device);
            NB_CUDA(cudaMalloc(&d, sizeof(int4) * v.size()));
            NB_CUDA(cudaMemcpy(d, v.data(), sizeof(int4) * v.size(), cudaMemcpyHostToDevice));
        }
        it = sp.box_lists.emplace(key, std::make_pair(d, (int64_t)v.size())).first;
    }
    *items = it->second.first;
    *n = it->second.second;
    return NB_OK;
}

static std::vector<int> spb_ranges(const nb_grid *g, int p, int which) {
    const NbPart &q = g->parts[p];
    const int nz = q.nz();
    if (which == 0) return {0, nz};
    const int ib = q.lo >= 0 ? 1 : 0, ie = std::max(ib, nz - (q.hi >= 0 ? 1 : 0));
    if (which == 1) return {ib, ie};
    std::vector<int> r;
    if (q.lo >= 0) r.insert(r.end(), {0, 1});
    if (q.hi >= 0 && ie < nz) r.insert(r.end(), {nz - 1, nz});
    return r;
}

// opt-in (NB_SP_CG_BOX=1): on the C4 sphere it measured 1.42 ms per iteration
// against 0.63 for the map / q / r segment schedule although it moves 40 %
// fewer bytes — it issues ~150 instructions per staged box cell (table
// lookups, 8-byte copies, the per-plane barrier and tile dot), and the
// sphere's boxes hold two cells per active one (ncu: 54 % issue, stalls at
// the plane barrier 28 % and on loads 25 %; prefetch depth 3 .. 10 planes
// made no difference).  On a full mask it gives the dense CG's bits.
bool nb_sparse_cg_boxed() { return getenv("NB_SP_CG_BOX") != nullptr; }

// tables, lists and the tile partial buffer (outside any graph capture)
nb_status nb_sparse_cg_box_prepare(nb_grid *g) {
    NB_TRY(nb_sparse_fem_box_tables(g));
    NB_TRY(nb_sparse_tile_tp(g));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p)
        for (int which = 0; which < 3; ++which) {
            const int4 *it;
            int64_t n;
            NB_TRY(spb_items(g, p, spb_ranges(g, p, which), &it, &n));
        }
    static unsigned attr_set = 0;  // per device: dynamic shared memory above 48 KB
    if (g->device >= 32 || !(attr_set & (1u << g->device))) {
        NB_CUDA(cudaFuncSetAttribute(k_sp_cg_box<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, SpbCfg<0>::SMEM));
        NB_CUDA(cudaFuncSetAttribute(k_sp_cg_box<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, SpbCfg<1>::SMEM));
        NB_CUDA(cudaFuncSetAttribute(k_sp_cg_box<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, SpbCfg<2>::SMEM));
        if (g->device < 32) attr_set |= 1u << g->device;
    }
    return NB_OK;
}

static nb_status spb_launch(nb_grid *g, int p, int ph, int which, SpCgBoxArgs A, const char *name) {
    const int4 *items;
    int64_t n;
    NB_TRY(spb_items(g, p, spb_ranges(g, p, which), &items, &n));
    if (n <= 0) return NB_OK;
    const NbSparsePart &sp = g->sp[p];
    A.items = items;
    A.rm = sp.d_rm;
    A.ri = sp.d_ri;
    A.rw = sp.rw;
    A.nx = g->nx;
    A.ny = g->ny;
    A.gz0 = g->parts[p].z0;
    A.nzl = g->parts[p].nz();
    A.NZ = g->nz;
    A.T = g->sp_T;
    A.tx = (g->nx + 31) / 32;
    A.tp = g->sp_tp;
    LaunchScope ls(g, g->cs, name);
    if (ph == 0)
        k_sp_cg_box<0><<<(unsigned)n, 256, SpbCfg<0>::SMEM, g->cs>>>(A);
    else if (ph == 1)
        k_sp_cg_box<1><<<(unsigned)n, 256, SpbCfg<1>::SMEM, g->cs>>>(A);
    else
        k_sp_cg_box<2><<<(unsigned)n, 256, SpbCfg<2>::SMEM, g->cs>>>(A);
    return nb_launch_check(name);
}

// set-up: r = b - A x0, rr0 (tile order)
static nb_status sp_cg_box_init(nb_cg *cg) {
    nb_grid *g = cg->g;
    NB_TRY(nb_sparse_cg_box_prepare(g));
    SpTpSwap sw(g);
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        SpCgBoxArgs A{};
        A.u = (const double *)cg->x->base[p];
        A.b = (const double *)cg->b->base[p];
        A.ro = (double *)cg->r->base[p];
        A.sc = cg->sc;
        NB_TRY(spb_launch(g, p, 2, 0, A, "k_sp_cg_init"));
    }
    return nb_reduce_finalize(g, 1, FIN_CG_INIT, cg->sc, 0);
}

// one iteration: p_new of the boundary planes facing a neighbour -> their
// halo (OCC: interior phase A while it flies) -> phase A -> alpha -> phase B
// -> beta
static nb_status sp_cg_box_iter(nb_cg *cg, int parity) {
    nb_grid *g = cg->g;
    nb_field *pn = cg->p[parity], *po = cg->p[parity ^ 1];
    const bool split = cg->prm.occ != NB_OCC_NONE && g->nparts > 1 && (nb_is_peer(g) || nb_halo_on_stream(g));
    SpTpSwap sw(g);
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p)
        NB_TRY(nb_sparse_pmap(g, p, 1, (const double *)po->base[p], (const double *)cg->r->base[p],
                              (double *)pn->base[p], cg->sc));
    auto phase_a = [&](int p, int which) {
        SpCgBoxArgs A{};
        A.u = (const double *)pn->base[p];
        A.r = (const double *)cg->r->base[p];
        A.po = (const double *)po->base[p];
        A.pn = (double *)pn->base[p];
        A.x = (double *)cg->x->base[p];
        A.sc = cg->sc;
        return spb_launch(g, p, 0, which, A, "k_sp_cg_a");
    };
    if (!split) {
        if (g->nparts > 1) NB_TRY(nb_sparse_halo_update(pn));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) NB_TRY(phase_a(p, 0));
    } else {
        NB_TRY(nb_halo_split_begin(pn, 0, 1, cg->hs));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) NB_TRY(phase_a(p, 1));
        NB_TRY(nb_halo_split_wait(g, cg->hs));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) NB_TRY(phase_a(p, 2));
    }
    NB_TRY(nb_reduce_finalize(g, 1, FIN_CG_PQ, cg->sc, 0));
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        SpCgBoxArgs A{};
        A.u = (const double *)pn->base[p];
        A.ro = (double *)cg->r->base[p];
        A.sc = cg->sc;
        NB_TRY(spb_launch(g, p, 1, 0, A, "k_sp_cg_b"));
    }
    NB_TRY(nb_reduce_finalize(g, 1, FIN_CG_RR, cg->sc, 0));
    cg->k += 1;
    return NB_OK;
}

__global__ void k_sp_cg_flush(double *x, const double *p0, const double *p1, int64_t n, const CgScal *sc) {
    if (!sc->pending) return;
    const double *p = (p1 && (sc->iters & 1)) ? p1 : p0;  // ping-pong: the last p_new
    const double a = sc->alpha_prev;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[i] = fma(a, p[i], x[i]);
}

nb_status nb_sparse_cg_flush(nb_cg *cg) {
    nb_grid *g = cg->g;
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbSparsePart &sp = g->sp[p];
        for (int c = 0; c < cg->x->card; ++c) {
            const int64_t o = (int64_t)c * cg->x->pcs[p] + sp.hl;
            LaunchScope ls(g, g->cs, "k_sp_cg_flush");
            k_sp_cg_flush<<<296, 256, 0, g->cs>>>((double *)cg->x->base[p] + o, (const double *)cg->p[0]->base[p] + o,
                                                  cg->pingpong ? (const double *)cg->p[1]->base[p] + o : nullptr,
                                                  sp.n, cg->sc);
            NB_TRY(nb_launch_check("k_sp_cg_flush"));
        }
    }
    return NB_OK;
}

// ===========================================================================
// FEM on element-sparse grids (the
// linear-elastic FEM on "dense and sparse" domains).  Nodes = active cells;
// an element exists iff its 8 nodes are active (the oracle's reading,
// oracle/oracle.c elem_exists).  The operator (nb_fem.cu k_sp_fem) needs each
// node's 27-neighbourhood: an activity mask and, per (y, z) row, the buffer
// index of the first active cell among x-1 .. x+1 (a row's active cells are
// consecutive in the (z, y, x) order), 40 B per node, built here once.
// ===========================================================================
__global__ void k_sp_fem_tab(const uint8_t *__restrict__ mask, const int32_t *__restrict__ map, int nx, int ny,
                             int slab_z0, int nslab, int z0, int hl, int64_t n, uint32_t *fm, int32_t *fb) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y, z = z0 + blockIdx.z;
    if (x >= nx) return;
    const int64_t plane = (int64_t)nx * ny;
    const int64_t cell = (int64_t)(z - slab_z0) * plane + (int64_t)y * nx + x;
    if (!mask[cell]) return;
    const int64_t j = (int64_t)map[cell] - hl;
    uint32_t m = 0;
#pragma unroll
    for (int r = 0; r < 9; ++r) {
        const int yy = y + r % 3 - 1, zz = z + r / 3 - 1 - slab_z0;
        int32_t base = -1;
        if (yy >= 0 && yy < ny && zz >= 0 && zz < nslab) {
            const int64_t row = (int64_t)zz * plane + (int64_t)yy * nx;
#pragma unroll
            for (int dx = -1; dx <= 1; ++dx) {
                const int xx = x + dx;
                if (xx < 0 || xx >= nx || !mask[row + xx]) continue;
                m |= 1u << (r * 3 + dx + 1);
                if (base < 0) base = map[row + xx];
            }
        }
        if (fb) fb[(int64_t)r * n + j] = base;
    }
    fm[j] = m;
}

nb_status nb_sparse_fem_tables(nb_grid *g, bool with_bases) {
    if (!g->sparse) return NB_OK;
    DeviceGuard dg(g->device);
    const int nx = g->nx, ny = g->ny;
    const int64_t plane = (int64_t)nx * ny;
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        NbSparsePart &sp = g->sp[p];
        if (sp.d_fm && (sp.d_fb || !with_bases)) continue;
        cudaFree(sp.d_fm);  // rebuilt with the row bases
        sp.d_fm = nullptr;
        const NbPart &q = g->parts[p];
        const int slab_z0 = q.z0 - (q.lo >= 0 ? 1 : 0), slab_z1 = q.z1 + (q.hi >= 0 ? 1 : 0);
        const int nslab = slab_z1 - slab_z0;
        const int64_t ncell = (int64_t)nslab * plane;
        uint8_t *d_mask = nullptr;
        int32_t *d_map = nullptr;
        void *tmp = nullptr;
        size_t tmp_bytes = 0;
        NB_CUDA(cudaMalloc(&sp.d_fm, sizeof(uint32_t) * std::max<int64_t>(sp.n, 1)));
        // the 9 row bases (36 B / node) only for the gather pass
        if (with_bases) NB_CUDA(cudaMalloc(&sp.d_fb, sizeof(int32_t) * 9 * std::max<int64_t>(sp.n, 1)));
        NB_CUDA(cudaMalloc(&d_mask, ncell));
        NB_CUDA(cudaMalloc(&d_map, ncell * 4));
        NB_CUDA(cudaMemcpyAsync(d_mask, g->host_mask.data() + (int64_t)slab_z0 * plane, ncell, cudaMemcpyHostToDevice,
                                g->cs));
        cub::TransformInputIterator<int, MaskToInt, const uint8_t *> it(d_mask, MaskToInt());
        cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, it, d_map, ncell, g->cs);
        NB_CUDA(cudaMalloc(&tmp, tmp_bytes));
        NB_CUDA(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, it, d_map, ncell, g->cs));
        if (q.nz() > 0 && sp.n > 0) {
            dim3 blk(128), grd((nx + 127) / 128, ny, q.nz());
            LaunchScope ls(g, g->cs, "k_sp_fem_tab");
            k_sp_fem_tab<<<grd, blk, 0, g->cs>>>(d_mask, d_map, nx, ny, slab_z0, nslab, q.z0, (int)sp.hl, sp.n, sp.d_fm,
                                                 sp.d_fb);
            NB_TRY(nb_launch_check("k_sp_fem_tab"));
        }
        NB_CUDA(cudaStreamSynchronize(g->cs));
        cudaFree(d_mask);
        cudaFree(d_map);
        cudaFree(tmp);
    }
    return NB_OK;
}

// Box tables of the shared-memory FEM operator (nb_fem.cu k_sp_fem_box):
// a CTA stages the 34 x 10 box of each plane around its 32 x 8 tile from the
// compact arrays.  A box cell's buffer index is that of its row word's first
// cell position plus the active cells before it in the word (a popcount), so
// per (slab row, 32-cell word) the table holds the activity bits and that
// index: 8 B per 32 cells, built here on the host from the mask.
nb_status nb_sparse_fem_box_tables(nb_grid *g) {
    if (!g->sparse) return NB_OK;
    DeviceGuard dg(g->device);
    const int nx = g->nx, ny = g->ny;
    const int64_t plane = (int64_t)nx * ny;
    const int rw = (nx + 31) / 32, tx = rw, ty = (ny + 7) / 8;
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        NbSparsePart &sp = g->sp[p];
        if (sp.d_rm) continue;
        const NbPart &q = g->parts[p];
        const int nzl = q.nz();
        if (sp.hl + sp.n + sp.hh >= ((int64_t)1 << 31))
            NB_FAIL(NB_EUNSUPPORTED, "sparse FEM box tables: more than 2^31 cells in a slab");
        const int64_t nrow = (int64_t)(nzl + 2) * ny;
        std::vector<uint32_t> rm((size_t)(nrow * rw), 0u);
        std::vector<int32_t> ri((size_t)(nrow * rw), 0);
        sp.tile_any.assign((size_t)nzl * ty * tx, 0);
        for (int s = 0; s < nzl + 2; ++s) {
            const int zl = s - 1, gz = q.z0 + zl;
            int64_t idx;
            if (zl == -1) {
                if (q.lo < 0) continue;
                idx = 0;
            } else if (zl == nzl) {
                if (q.hi < 0) continue;
                idx = sp.hl + sp.n;
            } else {
                idx = sp.hl + sp.pstart[zl];
            }
            const uint8_t *m = g->host_mask.data() + (int64_t)gz * plane;
            for (int y = 0; y < ny; ++y) {
                const uint8_t *row = m + (int64_t)y * nx;
                const int64_t k0 = ((int64_t)s * ny + y) * rw;
                for (int w = 0; w < rw; ++w) {
                    ri[k0 + w] = (int32_t)idx;
                    uint32_t bits = 0;
                    const int xe = std::min(nx, 32 * w + 32);
                    for (int x = 32 * w; x < xe; ++x)
                        if (row[x]) {
                            bits |= 1u << (x - 32 * w);
                            ++idx;
                        }
                    rm[k0 + w] = bits;
                    if (bits && zl >= 0 && zl < nzl) sp.tile_any[((size_t)zl * ty + y / 8) * tx + w] = 1;
                }
            }
        }
        // non-interior own nodes: interior = all 27 neighbours active (then
        // all 8 elements exist) and gz >= 2; the 3x3x3 erosion of the slab
        // mask, separable (x, then y, then z)
        std::vector<uint8_t> ex((size_t)(nzl + 2) * plane, 0), ey((size_t)(nzl + 2) * plane, 0);
        auto act = [&](int gz, int y, int x) -> bool {
            return gz >= 0 && gz < g->nz && y >= 0 && y < ny && x >= 0 && x < nx &&
                   g->host_mask[(size_t)gz * plane + (size_t)y * nx + x] != 0;
        };
        for (int s = 0; s < nzl + 2; ++s) {
            const int gz = q.z0 + s - 1;
            if (gz < 0 || gz >= g->nz) continue;
            for (int y = 0; y < ny; ++y)
                for (int x = 0; x < nx; ++x)
                    ex[(size_t)s * plane + (size_t)y * nx + x] = act(gz, y, x - 1) && act(gz, y, x) && act(gz, y, x + 1);
            for (int y = 0; y < ny; ++y)
                for (int x = 0; x < nx; ++x) {
                    const size_t c = (size_t)s * plane + (size_t)y * nx + x;
                    ey[c] = ex[c] && (y > 0 && ex[c - nx]) && (y + 1 < ny && ex[c + nx]);
                }
        }
        // buffer index of slab row (s, y) cell x (active), from the row tables
        auto bidx = [&](int s, int y, int x) -> int32_t {
            const int64_t k = ((int64_t)s * ny + y) * rw + (x >> 5);
            return ri[k] + __builtin_popcount(rm[k] & ((1u << (x & 31)) - 1u));
        };
        struct Node {  // nb_fem.cu SpFemNode
            int32_t i, gz;
            uint32_t m;
            int32_t base[9];
        };
        static_assert(sizeof(Node) == 48, "k_sp_fem_list reads 48-byte records");
        std::vector<Node> nodes;
        sp.fnode_start.assign(nzl + 1, 0);
        for (int zl = 0; zl < nzl; ++zl) {
            const int gz = q.z0 + zl;
            sp.fnode_start[zl] = (int64_t)nodes.size();
            for (int y = 0; y < ny; ++y)
                for (int x = 0; x < nx; ++x) {
                    if (!act(gz, y, x)) continue;
                    const size_t c = (size_t)y * nx + x;
                    const bool interior = gz >= 2 && ey[(size_t)zl * plane + c] && ey[(size_t)(zl + 1) * plane + c] &&
                                          ey[(size_t)(zl + 2) * plane + c];
                    if (interior) continue;
                    Node nd{};
                    nd.i = bidx(zl + 1, y, x);
                    nd.gz = gz;
                    for (int r = 0; r < 9; ++r) {
                        const int oy = r % 3 - 1, oz = r / 3 - 1;
                        nd.base[r] = -1;
                        for (int dx = -1; dx <= 1; ++dx)
                            if (act(gz + oz, y + oy, x + dx)) {
                                nd.m |= 1u << (3 * r + dx + 1);
                                if (nd.base[r] < 0) nd.base[r] = bidx(zl + 1 + oz, y + oy, x + dx);
                            }
                    }
                    nodes.push_back(nd);
                }
        }
        sp.fnode_start[nzl] = (int64_t)nodes.size();
        if (!nodes.empty()) {
            NB_CUDA(cudaMalloc(&sp.d_fnode, sizeof(Node) * nodes.size()));
            NB_CUDA(cudaMemcpy(sp.d_fnode, nodes.data(), sizeof(Node) * nodes.size(), cudaMemcpyHostToDevice));
        }
        NB_CUDA(cudaMalloc(&sp.d_rm, sizeof(uint32_t) * rm.size()));
        NB_CUDA(cudaMalloc(&sp.d_ri, sizeof(int32_t) * ri.size()));
        NB_CUDA(cudaMemcpy(sp.d_rm, rm.data(), sizeof(uint32_t) * rm.size(), cudaMemcpyHostToDevice));
        NB_CUDA(cudaMemcpy(sp.d_ri, ri.data(), sizeof(int32_t) * ri.size(), cudaMemcpyHostToDevice));
        sp.rw = rw;
    }
    return NB_OK;
}

// work items {tile x, tile y, zs, ze}: every (tile, chunk of <= zc planes) of
// the local plane ranges holding an active node, chunk-major (neighbouring
// tiles of a chunk run together and share their ring rows in L2); cached
nb_status nb_sparse_fem_box_list(nb_grid *g, int p, const std::vector<int> &ranges, int zc, const int4 **items,
                                 int64_t *n, bool all, int th) {
    NB_TRY(nb_sparse_fem_box_tables(g));
    NbSparsePart &sp = g->sp[p];
    std::vector<int> key = ranges;
    key.push_back(zc);
    key.push_back(all ? 1 : 0);
    key.push_back(th);
    auto it = sp.box_lists.find(key);
    if (it == sp.box_lists.end()) {
        // tile_any is per 32 x 8 tile; a 32 x th tile spans th / 8 of them
        const int tx = (g->nx + 31) / 32, ty = (g->ny + 7) / 8, f = th / 8, tyh = (ty + f - 1) / f;
        std::vector<int4> v;
        for (size_t r = 0; r + 1 < ranges.size(); r += 2)
            for (int zs = ranges[r]; zs < ranges[r + 1]; zs += zc) {
                const int ze = std::min(zs + zc, ranges[r + 1]);
                for (int by = 0; by < tyh; ++by)
                    for (int bx = 0; bx < tx; ++bx) {
                        bool any = false;
                        for (int zl = zs; zl < ze && !any; ++zl)
                            for (int k = 0; k < f && by * f + k < ty && !any; ++k)
                                any = sp.tile_any[((size_t)zl * ty + by * f + k) * tx + bx] != 0;
                        // all: every tile (its dot partials are rewritten), empty ones flagged
                        if (any || all) v.push_back(make_int4(bx | (any ? 0 : 0x40000000), by, zs, ze));
                    }
            }
        int4 *d = nullptr;
        if (!v.empty()) {
            DeviceGuard dg(g->device);
            NB_CUDA(cudaMalloc(&d, sizeof(int4) * v.size()));
            NB_CUDA(cudaMemcpy(d, v.data(), sizeof(int4) * v.size(), cudaMemcpyHostToDevice));
        }
        it = sp.box_lists.emplace(key, std::make_pair(d, (int64_t)v.size())).first;
    }
    *items = it->second.first;
    *n = it->second.second;
    return NB_OK;
}

// tile partials of the box kernels' dots: [3 components][nz][sp_T], sp_T =
// the 32 x 8 tiles of a plane (the dense canonical order); lazy
nb_status nb_sparse_tile_tp(nb_grid *g) {
    if (g->sp_tp) return NB_OK;
    DeviceGuard dg(g->device);
    g->sp_T = ((g->nx + 31) / 32) * ((g->ny + 7) / 8);
    const size_t n = (size_t)3 * g->nz * g->sp_T;
    NB_CUDA(cudaMalloc(&g->sp_tp, sizeof(double) * n));
    NB_CUDA(cudaMemset(g->sp_tp, 0, sizeof(double) * n));
    return NB_OK;
}

// consistent nodal load of pressure pr on the exposed top faces (+z) of the
// existing elements (oracle or_fem_rhs with a mask): a node gets pr/4 from
// each existing element below it whose top face is exposed (no existing
// element above), Dirichlet (z = 0) nodes none.  Element tests use the
// 27-neighbourhood mask: element with lower corner node + (dx, dy, dz)
__device__ __forceinline__ bool sp_fem_elem(uint32_t m, int dx, int dy, int dz) {
#pragma unroll
    for (int b = 0; b < 8; ++b) {
        const int ox = dx + (b & 1), oy = dy + ((b >> 1) & 1), oz = dz + ((b >> 2) & 1);
        if (ox < -1 || ox > 1 || oy < -1 || oy > 1 || oz < -1 || oz > 1) return false;
        if (!((m >> ((ox + 1) + 3 * (oy + 1) + 9 * (oz + 1))) & 1u)) return false;
    }
    return true;
}

__global__ void k_sp_fem_rhs(const int32_t *__restrict__ seg, int64_t nseg, const int64_t *__restrict__ pstart,
                             const uint32_t *__restrict__ fm, int64_t hl, int64_t cs, int gz0, double pr, double *b) {
    const int64_t q = blockIdx.x;
    if (q >= nseg) return;
    const int e = seg[q], zl = e >> 16;
    const int64_t j = pstart[zl] + (int64_t)(e & 0xffff) * SEG + threadIdx.x;
    if (j >= pstart[zl + 1]) return;
    const int gz = gz0 + zl;
    const uint32_t m = fm[j];
    double v = 0.0;
    if (gz > 0) {
        // elements below (dz = -1) having this node as a top corner, exposed
        // when the element above them (dz = 0, same dx, dy) does not exist;
        // added in the oracle's element order (ey, then ex)
        for (int dy = -1; dy <= 0; ++dy)
            for (int dx = -1; dx <= 0; ++dx)
                if (sp_fem_elem(m, dx, dy, -1) && !sp_fem_elem(m, dx, dy, 0)) v = v + 0.25 * pr;
    }
    b[0 * cs + hl + j] = 0.0;
    b[1 * cs + hl + j] = 0.0;
    b[2 * cs + hl + j] = v;
}

nb_status nb_sparse_fem_rhs(nb_field *b, double pr) {
    nb_grid *g = b->g;
    NB_TRY(nb_sparse_fem_tables(g, false));  // the masks only
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbSparsePart &sp = g->sp[p];
        const int64_t nseg = sp.seg_start.back();
        if (nseg <= 0) continue;
        LaunchScope ls(g, g->cs, "k_fem_rhs");
        k_sp_fem_rhs<<<(unsigned)nseg, SEG, 0, g->cs>>>(sp.d_seg, nseg, sp.d_pstart, sp.d_fm, sp.hl, b->pcs[p],
                                                       g->parts[p].z0, pr, (double *)b->base[p]);
        NB_TRY(nb_launch_check("k_sp_fem_rhs"));
    }
    return NB_OK;
}

// sparse FEM CG: map (x deferred update, p = r + beta p) per component ->
// halo(p, 3 components) -> q = K p, <p, q> -> alpha -> r -= alpha q, <r, r>
// per component -> beta (the Poisson sparse schedule with the FEM operator;
// OCC as there: boundary map, halo in flight with the interior map / K p,
// boundary K p after the wait)
nb_status nb_sparse_fem_cg_hooks(nb_cg *cg, int parity) {
    nb_grid *g = cg->g;
    const nb_occ occ = cg->prm.occ;
    const bool split = occ != NB_OCC_NONE && g->nparts > 1 && (nb_is_peer(g) || nb_halo_on_stream(g));
    if (cg->pingpong) {
        // fused phase A (the dense FEM CG's schedule on the sparse grid):
        // p_new of the boundary planes facing a neighbour -> their halo ->
        // phase A (p_new, deferred x, q = K p_new; interior planes while the
        // halo flies) -> the list nodes' q -> <p_new, q> -> alpha -> r -> beta.
        // Same values as the map + q schedule below (bitwise).
        nb_field *pn = cg->p[parity], *po = cg->p[parity ^ 1];
        auto cga = [&](int p) {
            return SpFemCgA{(const double *)cg->r->base[p], (const double *)po->base[p], (double *)pn->base[p],
                            (double *)cg->x->base[p]};
        };
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p)
            NB_TRY(nb_sparse_pmap(g, p, 3, (const double *)po->base[p], (const double *)cg->r->base[p],
                                  (double *)pn->base[p], cg->sc));
        auto phase_a = [&](int p, int which) {
            const SpFemCgA c = cga(p);
            return nb_sparse_fem_box_ranges(g, p, which, nullptr, nullptr, (double *)cg->q->base[p], cg->sc, 3, &c);
        };
        if (!split) {
            if (g->nparts > 1) NB_TRY(nb_sparse_halo_update(pn));
            for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) NB_TRY(phase_a(p, 0));
        } else {
            NB_TRY(nb_halo_split_begin(pn, 0, 3, cg->hs));
            for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) NB_TRY(phase_a(p, 1));
            NB_TRY(nb_halo_split_wait(g, cg->hs));
            for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) NB_TRY(phase_a(p, 2));
        }
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p)
            NB_TRY(nb_sparse_fem_dot(g, p, (const double *)pn->base[p], (const double *)cg->q->base[p], cg->sc));
        NB_TRY(nb_reduce_finalize(g, 3, FIN_CG_PQ, cg->sc, 0));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p)
            for (int c = 0; c < 3; ++c) {
                SpArgs A{};
                const int64_t o = (int64_t)c * pn->pcs[p];
                A.a = (const double *)cg->q->base[p] + o;
                A.c = (double *)cg->r->base[p] + o;
                A.sc = cg->sc;
                NB_TRY(sp_launch<SPK_CG_R>(g, p, 0, g->parts[p].nz(), A, c * g->nz, "k_sp_cg_r"));
            }
        NB_TRY(nb_reduce_finalize(g, 3, FIN_CG_RR, cg->sc, 0));
        cg->k += 1;
        return NB_OK;
    }
    nb_field *p_ = cg->p[0];
    auto map_args = [&](int p, int c) {
        SpArgs A{};
        const int64_t o = (int64_t)c * p_->pcs[p];
        A.a = (const double *)cg->r->base[p] + o;
        A.c = (double *)p_->base[p] + o;
        A.d = (double *)cg->x->base[p] + o;
        A.sc = cg->sc;
        return A;
    };
    auto qpass = [&](int p, const int32_t *list, const int32_t *gi, int64_t s0, int64_t n) {
        return nb_sparse_fem_pass(g, p, 1, list, gi, s0, n, (const double *)p_->base[p], nullptr,
                                  (double *)cg->q->base[p], cg->sc);
    };
    // box operator (default): q = K p over plane ranges (which: 0 all, 1
    // interior, 2 boundary planes), then <p, q> per segment in one pass
    const bool box = nb_sparse_fem_boxed();
    // <p, q> in a separate segment-order pass (default: the gather pass's
    // dot, so the box schedule is bitwise equal to it) or, with
    // NB_SPF_TILEDOT=1, inside the box kernel in tile order (into sp_tp; the
    // list nodes then run first, not concurrently): 3.19 against 3.28 ms per
    // iteration on the full 384^3 cube but 1.24 against 1.22 on the sphere
    const bool segdot = box && !getenv("NB_SPF_TILEDOT");
    auto qbox = [&](int p, int which) {
        return nb_sparse_fem_box_ranges(g, p, which, (const double *)p_->base[p], nullptr, (double *)cg->q->base[p],
                                        cg->sc, segdot ? 0 : 1, nullptr);
    };
    auto qdot = [&]() -> nb_status {
        if (segdot)
            for (int p = g->first_local; p < g->first_local + g->nlocal; ++p)
                NB_TRY(nb_sparse_fem_dot(g, p, (const double *)p_->base[p], (const double *)cg->q->base[p], cg->sc));
        return NB_OK;
    };
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const NbSparsePart &sp = g->sp[p];
        for (int c = 0; c < 3; ++c) {
            if (split)
                NB_TRY(sp_launch_list<SPK_CG_MAP>(g, p, sp.d_seg_bnd, sp.n_seg_bnd, map_args(p, c), 0, "k_sp_cg_map"));
            else
                NB_TRY(sp_launch<SPK_CG_MAP>(g, p, 0, g->parts[p].nz(), map_args(p, c), 0, "k_sp_cg_map"));
        }
    }
    if (!split) {
        NB_TRY(nb_sparse_halo_update(p_));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            const NbSparsePart &sp = g->sp[p];
            NB_TRY(box ? qbox(p, 0) : qpass(p, sp.d_seg, nullptr, 0, sp.seg_start.back()));
        }
    } else {
        NB_TRY(nb_halo_split_begin(p_, 0, 3, cg->hs));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            const NbPart &q = g->parts[p];
            const NbSparsePart &sp = g->sp[p];
            const int ib = q.lo >= 0 ? 1 : 0, ie = std::max(ib, q.nz() - (q.hi >= 0 ? 1 : 0));
            for (int c = 0; c < 3; ++c)
                NB_TRY(sp_launch<SPK_CG_MAP>(g, p, ib, ie, map_args(p, c), 0, "k_sp_cg_map"));
            NB_TRY(box ? qbox(p, 1) : qpass(p, sp.d_seg, nullptr, sp.seg_start[ib], sp.seg_start[ie] - sp.seg_start[ib]));
        }
        NB_TRY(nb_halo_split_wait(g, cg->hs));
        for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
            const NbSparsePart &sp = g->sp[p];
            NB_TRY(box ? qbox(p, 2) : qpass(p, sp.d_seg_bnd, sp.d_seg_bnd_gi, 0, sp.n_seg_bnd));
        }
    }
    NB_TRY(qdot());
    if (box && !segdot) {
        SpTpSwap sw(g);
        NB_TRY(nb_reduce_finalize(g, 3, FIN_CG_PQ, cg->sc, 0));
    } else {
        NB_TRY(nb_reduce_finalize(g, 3, FIN_CG_PQ, cg->sc, 0));
    }
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p)
        for (int c = 0; c < 3; ++c) {
            SpArgs A{};
            const int64_t o = (int64_t)c * p_->pcs[p];
            A.a = (const double *)cg->q->base[p] + o;
            A.c = (double *)cg->r->base[p] + o;
            A.sc = cg->sc;
            NB_TRY(sp_launch<SPK_CG_R>(g, p, 0, g->parts[p].nz(), A, c * g->nz, "k_sp_cg_r"));
        }
    NB_TRY(nb_reduce_finalize(g, 3, FIN_CG_RR, cg->sc, 0));
    cg->k += 1;
    return NB_OK;
}
