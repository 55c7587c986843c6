// nb_api.cu — grid, field, halo, map and reduce entry points of libnb.
//
// Paper: Neon (Meneghin et al., IPDPS 2022), /root/reference/PAPER.md.
//   Grid / Field / views / haloUpdate: §IV-C
//   MapOp / ReduceOp:                  §III-b L96-L131 (eqs.)
//   Host logical view:                 L219-L221
// Design: DESIGN.md ("Data layout", "Deterministic reductions", "Halo").
#include <dlfcn.h>

#include <algorithm>
#include <cstdarg>
#include <cstring>
#include <mutex>

#include "nb_device.cuh"
#include "nb_internal.cuh"
#include "nb_zmarch.cuh"

// ===========================================================================
// errors, version
// ===========================================================================
static thread_local char g_err[1024] = "";

void nb_set_error(const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
}

extern "C" const char *nb_version(void) { return "nb 0.1.0 (sm_100a)"; }
extern "C" const char *nb_last_error(void) { return g_err; }

extern "C" int32_t nb_device_count(void) {
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return n;
}

nb_status nb_launch_check(const char *what) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) NB_FAIL(NB_ECUDA, "launch of %s failed: %s", what, cudaGetErrorString(e));
    return NB_OK;
}


// ===========================================================================
// NCCL, loaded at run time (no link-time dependency; one process per GPU)
// ===========================================================================
namespace {
typedef int nccl_res_t;
struct NcclApi {
    void *h = nullptr;
    nccl_res_t (*GetUniqueId)(void *id) = nullptr;
    nccl_res_t (*CommInitRank)(void **comm, int nranks, /*ncclUniqueId by value*/ ...) = nullptr;
    nccl_res_t (*CommDestroy)(void *comm) = nullptr;
    nccl_res_t (*Send)(const void *, size_t, int, int, void *, cudaStream_t) = nullptr;
    nccl_res_t (*Recv)(void *, size_t, int, int, void *, cudaStream_t) = nullptr;
    nccl_res_t (*AllReduce)(const void *, void *, size_t, int, int, void *, cudaStream_t) = nullptr;
    nccl_res_t (*GroupStart)() = nullptr;
    nccl_res_t (*GroupEnd)() = nullptr;
    const char *(*GetErrorString)(nccl_res_t) = nullptr;
};
struct NcclUid {
    char internal[128];
};
typedef nccl_res_t (*InitRankFn)(void **, int, NcclUid, int);
NcclApi g_nccl;
InitRankFn g_nccl_init = nullptr;
std::mutex g_nccl_mu;
constexpr int NCCL_UINT8 = 1, NCCL_FLOAT64 = 8, NCCL_SUM = 0;

nb_status nccl_load() {
    std::lock_guard<std::mutex> lk(g_nccl_mu);
    if (g_nccl.h) return NB_OK;
    const char *names[] = {"libnccl.so.2", "libnccl.so"};
    void *h = nullptr;
    for (const char *n : names)
        if ((h = dlopen(n, RTLD_NOW | RTLD_GLOBAL))) break;
    if (!h) {
        // the torch-bundled NCCL of the venv
        const char *env = getenv("NB_NCCL_LIB");
        if (env) h = dlopen(env, RTLD_NOW | RTLD_GLOBAL);
    }
    if (!h) NB_FAIL(NB_ENCCL, "cannot dlopen libnccl.so.2 (set NB_NCCL_LIB)");
#define LOAD(field, sym)                                                         \
    *(void **)(&g_nccl.field) = dlsym(h, sym);                                   \
    if (!g_nccl.field) NB_FAIL(NB_ENCCL, "libnccl is missing symbol %s", sym);
    LOAD(GetUniqueId, "ncclGetUniqueId");
    LOAD(CommDestroy, "ncclCommDestroy");
    LOAD(Send, "ncclSend");
    LOAD(Recv, "ncclRecv");
    LOAD(AllReduce, "ncclAllReduce");
    LOAD(GroupStart, "ncclGroupStart");
    LOAD(GroupEnd, "ncclGroupEnd");
    LOAD(GetErrorString, "ncclGetErrorString");
#undef LOAD
    *(void **)(&g_nccl_init) = dlsym(h, "ncclCommInitRank");
    if (!g_nccl_init) NB_FAIL(NB_ENCCL, "libnccl is missing ncclCommInitRank");
    g_nccl.h = h;
    return NB_OK;
}

#define NB_NCCL(call)                                                                   \
    do {                                                                                \
        nccl_res_t _r = (call);                                                         \
        if (_r != 0)                                                                    \
            NB_FAIL(NB_ENCCL, "%s failed: %s", #call,                                   \
                    g_nccl.GetErrorString ? g_nccl.GetErrorString(_r) : "?");           \
    } while (0)
}  // namespace

extern "C" nb_status nb_comm_unique_id(uint8_t out[128]) {
    if (!out) NB_FAIL(NB_EINVAL, "nb_comm_unique_id: out is NULL");
    NB_TRY(nccl_load());
    NcclUid id;
    NB_NCCL(g_nccl.GetUniqueId(&id));
    memcpy(out, id.internal, 128);
    return NB_OK;
}

extern "C" nb_status nb_comm_create(int32_t world, int32_t rank, const uint8_t id[128],
                                    int32_t device, nb_comm **out) {
    if (!out || !id || world < 1 || rank < 0 || rank >= world)
        NB_FAIL(NB_EINVAL, "nb_comm_create: bad arguments (world %d rank %d)", world, rank);
    *out = nullptr;
    if (device < 0 || device >= nb_device_count())
        NB_FAIL(NB_ECUDA, "nb_comm_create: device %d not available", device);
    nb_comm *c = new nb_comm();
    c->world = world;
    c->rank = rank;
    c->device = device;
    if (world > 1) {
        nb_status s = nccl_load();
        if (s != NB_OK) {
            delete c;
            return s;
        }
        DeviceGuard dg(device);
        NcclUid uid;
        memcpy(uid.internal, id, 128);
        nccl_res_t r = g_nccl_init(&c->nccl, world, uid, rank);
        if (r != 0) {
            delete c;
            NB_FAIL(NB_ENCCL, "ncclCommInitRank failed: %s", g_nccl.GetErrorString(r));
        }
    }
    *out = c;
    return NB_OK;
}

extern "C" nb_status nb_comm_destroy(nb_comm *comm) {
    if (!comm) return NB_OK;
    if (comm->nccl) g_nccl.CommDestroy(comm->nccl);
    delete comm;
    return NB_OK;
}

nb_status nb_nccl_allreduce_sum(nb_grid *g, const double *send, double *recv, size_t n,
                                cudaStream_t s) {
    NB_NCCL(g_nccl.AllReduce(send, recv, n, NCCL_FLOAT64, NCCL_SUM, g->comm->nccl, s));
    return NB_OK;
}
nb_status nb_nccl_group(nb_grid *g, bool start) {
    (void)g;
    if (start)
        NB_NCCL(g_nccl.GroupStart());
    else
        NB_NCCL(g_nccl.GroupEnd());
    return NB_OK;
}
nb_status nb_nccl_send(nb_grid *g, const void *buf, size_t bytes, int peer, cudaStream_t s) {
    NB_NCCL(g_nccl.Send(buf, bytes, NCCL_UINT8, peer, g->comm->nccl, s));
    return NB_OK;
}
nb_status nb_nccl_recv(nb_grid *g, void *buf, size_t bytes, int peer, cudaStream_t s) {
    NB_NCCL(g_nccl.Recv(buf, bytes, NCCL_UINT8, peer, g->comm->nccl, s));
    return NB_OK;
}

int nb_part_owner(const nb_grid *g, int part) {
    if (!g->comm || g->comm->world <= 1) return 0;
    return part / (g->nparts / g->comm->world);
}

// ===========================================================================
// partition plans (a1) — pure host logic
// ===========================================================================
extern "C" nb_status nb_partition_plan(int32_t nz, int32_t nparts, int32_t *z_begin) {
    if (!z_begin || nparts < 1 || nz < 1) NB_FAIL(NB_EINVAL, "nb_partition_plan: bad arguments");
    if (nparts > nz) NB_FAIL(NB_EINVAL, "nb_partition_plan: %d partitions for %d planes", nparts, nz);
    int base = nz / nparts, rem = nz % nparts, z = 0;
    for (int g = 0; g < nparts; ++g) {
        z_begin[g] = z;
        z += base + (g < rem ? 1 : 0);
    }
    z_begin[nparts] = nz;
    return NB_OK;
}

extern "C" nb_status nb_partition_plan_weighted(int32_t nz, const int64_t *counts, int32_t nparts,
                                                int32_t *z_begin) {
    if (!z_begin || !counts || nparts < 1 || nz < 1 || nparts > nz)
        NB_FAIL(NB_EINVAL, "nb_partition_plan_weighted: bad arguments");
    int64_t total = 0;
    for (int z = 0; z < nz; ++z) {
        if (counts[z] < 0) NB_FAIL(NB_EINVAL, "nb_partition_plan_weighted: negative count");
        total += counts[z];
    }
    z_begin[0] = 0;
    int64_t pref = 0;
    int z = 0;
    for (int g = 1; g < nparts; ++g) {
        // target prefix for the end of partition g-1; __int128 avoids overflow
        __int128 target = (__int128)total * g;
        int zmin = z_begin[g - 1] + 1;          // non-empty slab
        int zmax = nz - (nparts - g);           // leave >= 1 plane per remaining part
        while (z < zmin) pref += counts[z++];
        while (z < zmax && (__int128)pref * nparts < target) pref += counts[z++];
        // step back one plane if that lands closer to the target
        if (z > zmin) {
            __int128 over = (__int128)pref * nparts - target;
            __int128 under = target - (__int128)(pref - counts[z - 1]) * nparts;
            if (over > 0 && under < over) pref -= counts[--z];
        }
        z_begin[g] = z;
    }
    z_begin[nparts] = nz;
    return NB_OK;
}

extern "C" nb_status nb_halo_plan(int32_t nz, int32_t nparts, int32_t world, int32_t rank, int32_t periodic,
                                   nb_halo_msg *out, int32_t cap, int32_t *count) {
    if (!count || nparts < 1 || world < 1 || nparts % world != 0 || rank < -1 || rank >= world)
        NB_FAIL(NB_EINVAL, "nb_halo_plan: bad arguments");
    std::vector<int32_t> zb(nparts + 1);
    NB_TRY(nb_partition_plan(nz, nparts, zb.data()));
    const int k = nparts / world;
    int n = 0;
    auto emit = [&](int src, int dst, int up) -> bool {
        int sr = src / k, dr = dst / k;
        if (rank != -1 && sr != rank && dr != rank) return true;
        if (out) {
            if (n >= cap) return false;
            nb_halo_msg &m = out[n];
            m.src_part = src;
            m.dst_part = dst;
            m.src_rank = sr;
            m.dst_rank = dr;
            m.src_plane = up ? zb[src + 1] - zb[src] - 1 : 0;
            m.dst_plane = up ? -1 : zb[dst + 1] - zb[dst];
            m.up = up;
        }
        ++n;
        return true;
    };
    for (int p = 0; p < nparts; ++p) {
        int q = p + 1;
        if (q == nparts) {
            if (!periodic) break;
            q = 0;
        }
        // pair (p below, q above): p's top -> q's low halo; q's bottom -> p's high halo
        if (!emit(p, q, 1) || !emit(q, p, 0)) NB_FAIL(NB_EINVAL, "nb_halo_plan: cap %d too small", cap);
    }
    *count = n;
    return NB_OK;
}

// Execute the halo messages of field f for this process: local messages are
// device copies, remote ones grouped NCCL send/recv on stream s.  comps(up)
// gives the component range [c0, c1) carried by up / down messages.
// ---------------------------------------------------------------------------
// batched device-local plane copies: up to MAX (dst, src, bytes) descriptors
// per launch, passed by value; blocks are dealt to descriptors by a prefix of
// block counts.  16-byte vectors when every address and size allows it, else
// 4-byte words (every field element is >= 4 bytes).
// ---------------------------------------------------------------------------

__global__ void __launch_bounds__(256) k_halo_copy(const __grid_constant__ CopyBatch cb) {
    // grid-stride over the chunks: a capped grid leaves most SMs to the
    // interior kernels the copy overlaps with (OCC)
    const uint32_t total = cb.bstart[cb.n];
    int d = 0;
    for (uint32_t b = blockIdx.x; b < total; b += gridDim.x) {
        while (d + 1 < cb.n && cb.bstart[d + 1] <= b) ++d;
        const uint64_t w0 = (uint64_t)(b - cb.bstart[d]) * CopyBatch::CHUNK;
        const uint64_t w1 = min(w0 + CopyBatch::CHUNK, cb.words[d]);
        if ((cb.vec >> d) & 1ull) {
            const uint4 *s = (const uint4 *)cb.src[d];
            uint4 *t = (uint4 *)cb.dst[d];
            for (uint64_t i = w0 + threadIdx.x; i < w1; i += 256) t[i] = __ldcs(s + i);
        } else {
            const uint32_t *s = (const uint32_t *)cb.src[d];
            uint32_t *t = (uint32_t *)cb.dst[d];
            for (uint64_t i = w0 + threadIdx.x; i < w1; i += 256) t[i] = __ldcs(s + i);
        }
    }
}

// blocks of a batched halo copy on the halo stream: at most
// NB_HALO_COPY_BLOCKS (default 128, under one block per SM) so the copy does
// not take every SM away from the interior kernels it is meant to overlap;
// on the compute stream (stream-ordered copies) the full grid
static uint32_t halo_copy_blocks() {
    static uint32_t cap = [] {
        const char *v = getenv("NB_HALO_COPY_BLOCKS");
        int c = v ? atoi(v) : 128;
        return (uint32_t)(c > 0 ? c : 128);
    }();
    return cap;
}

nb_status nb_launch_copy_batch(nb_grid *g, const CopyBatch &cb, cudaStream_t s) {
    if (!cb.n || !cb.bstart[cb.n]) return NB_OK;
    NB_TRY(nb_delay_launch(g, 8, s));
    LaunchScope ls(g, s, "k_halo_copy");
    const uint32_t blocks = s == g->cs ? cb.bstart[cb.n] : std::min(cb.bstart[cb.n], halo_copy_blocks());
    k_halo_copy<<<blocks, 256, 0, s>>>(cb);
    return nb_launch_check("k_halo_copy");
}

nb_status nb_halo_run(nb_field *f, bool periodic, int c0u, int c1u, int c0d, int c1d, cudaStream_t s) {
    return nb_halo_run_mode(f, periodic, c0u, c1u, c0d, c1d, s, NB_HALO_GENERIC);
}

nb_status nb_halo_run_mode(nb_field *f, bool periodic, int c0u, int c1u, int c0d, int c1d, cudaStream_t s,
                           int mode) {
    nb_grid *g = f->g;
    int world = g->comm ? g->comm->world : 1, rank = g->comm ? g->comm->rank : 0;
    int cnt = 0;
    NB_TRY(nb_halo_plan(g->nz, g->nparts, world, rank, periodic, nullptr, 0, &cnt));
    std::vector<nb_halo_msg> msgs(cnt);
    NB_TRY(nb_halo_plan(g->nz, g->nparts, world, rank, periodic, msgs.data(), cnt, &cnt));
    // the contiguous pieces of components [c0, c1) of plane zl (include/nb.h
    // layouts): SOA one per component; SOA_PLANE one for the range; AOS the
    // whole interleaved plane (all components, one transfer)
    auto pieces = [&](int p, int zl, int c0, int c1) {
        std::vector<std::pair<int64_t, int64_t>> v;  // (element offset, elements)
        if (c1 <= c0) return v;
        const int64_t z = (int64_t)(zl + 1) * f->ps * f->es;
        if (f->layout == NB_SOA)
            for (int c = c0; c < c1; ++c) v.push_back({(int64_t)c * nb_cstride(f, p) + z, f->plane});
        else if (f->layout == NB_SOA_PLANE)
            v.push_back({(int64_t)c0 * f->plane + z, (int64_t)(c1 - c0) * f->plane});
        else
            v.push_back({z, f->plane * f->card});
        return v;
    };
    if (nb_is_peer(g)) {
        // peer memory: a "ready" round (the neighbours finished reading the
        // halos about to be overwritten), my planes stored straight into the
        // neighbours' (IPC-mapped) halos, a "done" round (NB_HALO_SEND: the
        // copies and a signal only)
        if (mode == NB_HALO_GENERIC) NB_TRY(nb_peer_round(g, periodic, s));
        CopyBatch cb;
        for (auto &m : msgs) {
            if (m.src_rank != rank) continue;  // the sender writes
            int c0 = m.up ? c0u : c0d, c1 = m.up ? c1u : c1d;
            auto sp = pieces(m.src_part, m.src_plane, c0, c1), dp = pieces(m.dst_part, m.dst_plane, c0, c1);
            for (size_t k = 0; k < sp.size(); ++k) {
                if (cb.n == CopyBatch::MAX) {
                    NB_TRY(nb_launch_copy_batch(g, cb, s));
                    cb = CopyBatch();
                }
                cb.add(f->base[m.dst_part] + dp[k].first * f->esz, f->base[m.src_part] + sp[k].first * f->esz,
                       (size_t)sp[k].second * f->esz);
            }
        }
        if (cb.n) NB_TRY(nb_launch_copy_batch(g, cb, s));
        return mode == NB_HALO_GENERIC ? nb_peer_round(g, periodic, s) : nb_peer_signal(g, periodic, s);
    }
    bool remote = false;
    // every device-local plane of the exchange goes into ONE batched copy
    // launch (a per-plane cudaMemcpyAsync costs ~4 us of host enqueue each,
    // which serialised the halo stream behind the host on LBM's 5-population
    // messages)
    CopyBatch cb;
    for (auto &m : msgs) {
        int c0 = m.up ? c0u : c0d, c1 = m.up ? c1u : c1d;
        if (m.src_rank == rank && m.dst_rank == rank) {
            auto sp = pieces(m.src_part, m.src_plane, c0, c1), dp = pieces(m.dst_part, m.dst_plane, c0, c1);
            for (size_t k = 0; k < sp.size(); ++k) {
                if (cb.n == CopyBatch::MAX) {
                    NB_TRY(nb_launch_copy_batch(g, cb, s));
                    cb = CopyBatch();
                }
                cb.add(f->base[m.dst_part] + dp[k].first * f->esz, f->base[m.src_part] + sp[k].first * f->esz,
                       (size_t)sp[k].second * f->esz);
            }
        } else {
            remote = true;
        }
    }
    if (cb.n) NB_TRY(nb_launch_copy_batch(g, cb, s));
    if (!remote) return NB_OK;
    NB_TRY(nb_nccl_group(g, true));
    for (auto &m : msgs) {
        if (m.src_rank == rank && m.dst_rank == rank) continue;
        int c0 = m.up ? c0u : c0d, c1 = m.up ? c1u : c1d;
        if (m.src_rank == rank) {
            for (auto &pc : pieces(m.src_part, m.src_plane, c0, c1))
                NB_TRY(nb_nccl_send(g, f->base[m.src_part] + pc.first * f->esz, (size_t)pc.second * f->esz,
                                    m.dst_rank, s));
        } else {
            for (auto &pc : pieces(m.dst_part, m.dst_plane, c0, c1))
                NB_TRY(nb_nccl_recv(g, f->base[m.dst_part] + pc.first * f->esz, (size_t)pc.second * f->esz,
                                    m.src_rank, s));
        }
    }
    NB_TRY(nb_nccl_group(g, false));
    return NB_OK;
}

// ===========================================================================
// grid
// ===========================================================================
nb_status nb_grid_alloc_common(nb_grid *g) {
    DeviceGuard dg(g->device);
    NB_CUDA(cudaStreamCreateWithFlags(&g->cs, cudaStreamNonBlocking));
    // the halo stream runs at the highest priority: its copies are small and
    // sit on the critical path, so the block scheduler should start them as
    // soon as an SM frees up instead of behind the interior kernel's
    // remaining CTAs (OCC)
    int prio_lo = 0, prio_hi = 0;
    NB_CUDA(cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi));
    NB_CUDA(cudaStreamCreateWithPriority(&g->hs, cudaStreamNonBlocking, prio_hi));
    g->own_cs = g->own_hs = true;
    g->tiles_x = (g->nx + DOT_TX - 1) / DOT_TX;
    g->tiles_y = (g->ny + DOT_TY - 1) / DOT_TY;
    if (!g->sparse) g->T = g->tiles_x * g->tiles_y;  // sparse: set by the builder (segments per plane)
    size_t planes = (size_t)g->max_card * g->nz;
    NB_CUDA(cudaMalloc(&g->tp, sizeof(double) * planes * g->T));
    NB_CUDA(cudaMalloc(&g->psum, sizeof(double) * planes));
    NB_CUDA(cudaMalloc(&g->psum_send, sizeof(double) * planes));
    NB_CUDA(cudaMalloc(&g->dots, sizeof(double) * NB_DOT_SLOTS));
    NB_CUDA(cudaMalloc(&g->counter, sizeof(unsigned int) * 16));
    NB_CUDA(cudaMemset(g->tp, 0, sizeof(double) * planes * g->T));
    NB_CUDA(cudaMemset(g->psum, 0, sizeof(double) * planes));
    NB_CUDA(cudaMemset(g->psum_send, 0, sizeof(double) * planes));
    NB_CUDA(cudaMemset(g->dots, 0, sizeof(double) * NB_DOT_SLOTS));
    NB_CUDA(cudaMemset(g->counter, 0, sizeof(unsigned int) * 16));
    if (nb_is_peer(g)) NB_TRY(nb_peer_grid_setup(g));  // collective
    return NB_OK;
}

nb_status nb_grid_setup_parts(nb_grid *g, const int32_t *zb, int32_t nparts,
                              const int32_t *device_ids, nb_comm *comm) {
    g->nparts = nparts;
    g->comm = comm;
    int world = comm ? comm->world : 1, rank = comm ? comm->rank : 0;
    if (nparts % world != 0)
        NB_FAIL(NB_EINVAL, "nparts (%d) must be a multiple of the world size (%d)", nparts, world);
    int k = nparts / world;
    g->first_local = rank * k;
    g->nlocal = k;
    g->parts.resize(nparts);
    for (int p = 0; p < nparts; ++p) {
        NbPart &q = g->parts[p];
        q.z0 = zb[p];
        q.z1 = zb[p + 1];
        q.lo = p > 0 ? p - 1 : -1;
        q.hi = p < nparts - 1 ? p + 1 : -1;
        q.local = (p >= g->first_local && p < g->first_local + k);
    }
    if (comm) {
        g->device = comm->device;
    } else {
        if (!device_ids) NB_FAIL(NB_EINVAL, "device_ids is NULL");
        g->device = device_ids[0];
        for (int p = 0; p < nparts; ++p)
            if (device_ids[p] != g->device)
                NB_FAIL(NB_EUNSUPPORTED,
                        "single-process grids keep all partitions on one device (got %d and %d); "
                        "use one process per GPU with an nb_comm",
                        g->device, device_ids[p]);
    }
    for (int p = 0; p < nparts; ++p) g->parts[p].device = g->device;
    if (g->device < 0 || g->device >= nb_device_count())
        NB_FAIL(NB_ECUDA, "CUDA device %d not available (no CPU fallback)", g->device);
    return NB_OK;
}

extern "C" nb_status nb_grid_create_dense(const int32_t dims[3], int32_t nparts,
                                          const int32_t *device_ids, nb_comm *comm,
                                          nb_grid **out) {
    if (!out || !dims) NB_FAIL(NB_EINVAL, "nb_grid_create_dense: NULL argument");
    *out = nullptr;
    if (dims[0] < 1 || dims[1] < 1 || dims[2] < 1 || dims[0] > 65535 || dims[1] > 65535)
        NB_FAIL(NB_EINVAL, "nb_grid_create_dense: bad dims %d x %d x %d", dims[0], dims[1], dims[2]);
    std::vector<int32_t> zb(nparts > 0 ? nparts + 1 : 1);
    NB_TRY(nb_partition_plan(dims[2], nparts, zb.data()));
    if (nparts > 1)
        for (int p = 0; p < nparts; ++p)
            if (zb[p + 1] - zb[p] < 2)
                NB_FAIL(NB_EUNSUPPORTED, "slab %d has %d plane(s); need >= 2 (radius 1)", p,
                        zb[p + 1] - zb[p]);
    nb_grid *g = new nb_grid();
    g->nx = dims[0];
    g->ny = dims[1];
    g->nz = dims[2];
    nb_status s = nb_grid_setup_parts(g, zb.data(), nparts, device_ids, comm);
    if (s == NB_OK) s = nb_grid_alloc_common(g);
    if (s != NB_OK) {
        nb_grid_destroy(g);
        return s;
    }
    for (auto &p : g->parts) {
        int64_t plane = (int64_t)g->nx * g->ny;
        p.n_act = plane * p.nz();
        p.n_lo_bnd = p.lo >= 0 ? plane : 0;
        p.n_hi_bnd = p.hi >= 0 ? plane : 0;
    }
    *out = g;
    return NB_OK;
}

void nb_sparse_free(nb_grid *g);  // nb_sparse.cu

nb_status nb_grid_scratch(nb_grid *g, nb_dtype dt, int card, int slot, nb_field **out) {
    auto key = std::make_pair((int)dt * 1000 + card, slot);
    auto it = g->scratch.find(key);
    if (it != g->scratch.end()) {
        *out = it->second;
        return NB_OK;
    }
    nb_field *f = nullptr;
    NB_TRY(nb_field_create(g, dt, card, NB_SOA, 0.0, &f));
    g->nfields--;  // owned by the grid
    g->scratch[key] = f;
    *out = f;
    return NB_OK;
}

extern "C" nb_status nb_grid_destroy(nb_grid *g) {
    if (!g) return NB_OK;
    if (g->nfields > 0 || g->nsolvers > 0)
        NB_FAIL(NB_ESTATE, "nb_grid_destroy: %d field(s) and %d solver(s) still alive", g->nfields,
                g->nsolvers);
    DeviceGuard dg(g->device);
    if (g->cs) cudaStreamSynchronize(g->cs);
    if (g->hs) cudaStreamSynchronize(g->hs);
    for (auto &kv : g->scratch) {
        g->nfields++;
        nb_field_destroy(kv.second);
    }
    g->scratch.clear();
    nb_field_cache_clear(g);
    if (g->c1_exec) cudaGraphExecDestroy(g->c1_exec);
    cudaFree(g->c1_tp);
    cudaFree(g->c1_psum);
    cudaFree(g->sp_tp);
    nb_peer_grid_teardown(g);  // collective (peer transport)
    for (auto &r : g->prof) {
        cudaEventDestroy(r.a);
        cudaEventDestroy(r.b);
    }
    nb_sparse_free(g);
    cudaFree(g->tp);
    cudaFree(g->psum);
    cudaFree(g->psum_send);
    cudaFree(g->dots);
    cudaFree(g->counter);
    if (g->own_cs && g->cs) cudaStreamDestroy(g->cs);
    if (g->own_hs && g->hs) cudaStreamDestroy(g->hs);
    if (g->fs) cudaStreamDestroy(g->fs);
    for (auto &e : g->fev)
        if (e) cudaEventDestroy(e);
    delete g;
    return NB_OK;
}

extern "C" nb_status nb_grid_num_partitions(const nb_grid *g, int32_t *n) {
    if (!g || !n) NB_FAIL(NB_EINVAL, "NULL argument");
    *n = g->nparts;
    return NB_OK;
}

extern "C" nb_status nb_grid_partition_info(const nb_grid *g, int32_t p, nb_part_info *o) {
    if (!g || !o || p < 0 || p >= g->nparts) NB_FAIL(NB_EINVAL, "nb_grid_partition_info: bad arguments");
    const NbPart &q = g->parts[p];
    o->device = q.device;
    o->local = q.local;
    o->z_begin = q.z0;
    o->z_end = q.z1;
    o->n_cells = q.n_act;
    o->n_bnd_lo = q.n_lo_bnd;
    o->n_bnd_hi = q.n_hi_bnd;
    o->n_internal = q.n_act - q.n_lo_bnd - (q.nz() > 1 ? q.n_hi_bnd : 0);
    return NB_OK;
}

extern "C" nb_status nb_grid_set_streams(nb_grid *g, void *cs, void *hs) {
    if (!g) NB_FAIL(NB_EINVAL, "NULL grid");
    DeviceGuard dg(g->device);
    if (cs) {
        if (g->own_cs) {
            cudaStreamSynchronize(g->cs);
            cudaStreamDestroy(g->cs);
        }
        g->cs = (cudaStream_t)cs;
        g->own_cs = false;
    }
    if (hs) {
        if (g->own_hs) {
            cudaStreamSynchronize(g->hs);
            cudaStreamDestroy(g->hs);
        }
        g->hs = (cudaStream_t)hs;
        g->own_hs = false;
    }
    return NB_OK;
}

extern "C" nb_status nb_grid_get_stream(const nb_grid *g, void **cs) {
    if (!g || !cs) NB_FAIL(NB_EINVAL, "NULL argument");
    *cs = (void *)g->cs;
    return NB_OK;
}

extern "C" nb_status nb_grid_set_halo_mode(nb_grid *g, int32_t mode) {
    if (!g) NB_FAIL(NB_EINVAL, "NULL grid");
    if (mode != NB_HALO_FUSED && mode != NB_HALO_STREAM) NB_FAIL(NB_EINVAL, "bad halo mode %d", mode);
    g->halo_mode = mode;
    return NB_OK;
}

extern "C" nb_status nb_sync(nb_grid *g) {
    if (!g) NB_FAIL(NB_EINVAL, "NULL grid");
    DeviceGuard dg(g->device);
    NB_CUDA(cudaStreamSynchronize(g->hs));
    NB_CUDA(cudaStreamSynchronize(g->cs));
    NB_CUDA(cudaGetLastError());
    return NB_OK;
}

extern "C" nb_status nb_grid_trim(nb_grid *g, int64_t *freed_bytes) {
    if (!g) NB_FAIL(NB_EINVAL, "NULL grid");
    DeviceGuard dg(g->device);
    NB_CUDA(cudaStreamSynchronize(g->hs));
    NB_CUDA(cudaStreamSynchronize(g->cs));
    int64_t n = 0;
    for (auto &kv : g->fcache) n += (int64_t)kv.first;
    nb_field_cache_clear(g);
    if (freed_bytes) *freed_bytes = n;
    return NB_OK;
}

// ===========================================================================
// fields (dense)
// ===========================================================================
nb_status nb_sparse_field_alloc(nb_field *f);            // nb_sparse.cu
nb_status nb_sparse_upload(nb_field *f, const void *host);
nb_status nb_sparse_download(const nb_field *f, void *host);
nb_status nb_sparse_fill(nb_field *f, nb_fill kind, uint64_t seed, double a, double b);

template <typename T>
__global__ void k_fill_const(T *p, int64_t n, T v) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x)
        p[i] = v;
}

static nb_status fill_const_raw(nb_grid *g, void *p, int64_t n, nb_dtype dt, double v,
                                cudaStream_t s) {
    if (n <= 0) return NB_OK;
    int blocks = (int)std::min<int64_t>((n + 255) / 256, 148 * 16);
    LaunchScope ls(g, s, "k_fill_const");
    if (dt == NB_F64)
        k_fill_const<double><<<blocks, 256, 0, s>>>((double *)p, n, v);
    else
        k_fill_const<float><<<blocks, 256, 0, s>>>((float *)p, n, (float)v);
    return nb_launch_check("k_fill_const");
}

static int64_t dense_pitch(const nb_grid *g) { return ((int64_t)g->nx + 31) / 32 * 32; }

// layout geometry of a dense field (include/nb.h layouts; nb_field)
static nb_status set_layout(nb_field *f, nb_layout layout) {
    if (layout < NB_SOA || layout > NB_AOS) NB_FAIL(NB_EINVAL, "bad layout %d", (int)layout);
    if (f->g->sparse && layout != NB_SOA && f->card > 1)
        NB_FAIL(NB_EUNSUPPORTED, "element-sparse grids store fields as SoA");
    f->layout = f->card == 1 ? NB_SOA : layout;  // one component: the layouts coincide
    if (f->g->sparse) return NB_OK;
    f->pitch = dense_pitch(f->g);
    f->plane = f->pitch * f->g->ny;
    f->es = f->layout == NB_AOS ? f->card : 1;
    f->ps = f->layout == NB_SOA_PLANE ? f->card * f->plane : f->plane;
    return NB_OK;
}

extern "C" nb_status nb_field_layout(const nb_field *f, nb_layout *layout) {
    if (!f || !layout) NB_FAIL(NB_EINVAL, "nb_field_layout: NULL argument");
    *layout = f->layout;
    return NB_OK;
}

// ---- field buffer cache -----------------------------------------------------
static bool field_cache_on(const nb_grid *g) {
    // single process only: across processes the buffers are IPC-exported and
    // mapped by the neighbours per field
    return !nb_is_peer(g) && !(g->comm && g->comm->world > 1) && !getenv("NB_NO_FIELD_CACHE");
}

void nb_field_cache_clear(nb_grid *g) {
    for (auto &kv : g->fcache) cudaFree(kv.second);
    g->fcache.clear();
}

nb_status nb_field_buf_alloc(nb_grid *g, size_t bytes, void **out) {
    *out = nullptr;
    auto it = g->fcache.find(bytes);
    if (it != g->fcache.end()) {
        *out = it->second;
        g->fcache.erase(it);
        return NB_OK;
    }
    cudaError_t e = cudaMalloc(out, bytes);
    if (e != cudaSuccess && !g->fcache.empty()) {  // give the cached buffers back and retry
        cudaGetLastError();
        nb_field_cache_clear(g);
        e = cudaMalloc(out, bytes);
    }
    if (e != cudaSuccess) {
        cudaGetLastError();
        *out = nullptr;
        NB_FAIL(NB_ENOMEM, "nb_field_create: cudaMalloc(%zu) failed: %s", bytes, cudaGetErrorString(e));
    }
    return NB_OK;
}

void nb_field_buf_release(nb_grid *g, void *buf, size_t bytes) {
    if (!buf) return;
    if (field_cache_on(g))
        g->fcache.emplace(bytes, buf);
    else
        cudaFree(buf);
}

extern "C" nb_status nb_field_create(nb_grid *g, nb_dtype dt, int32_t card, nb_layout layout, double outside,
                                     nb_field **out) {
    if (!g || !out) NB_FAIL(NB_EINVAL, "nb_field_create: NULL argument");
    *out = nullptr;
    if (dt != NB_F32 && dt != NB_F64) NB_FAIL(NB_EINVAL, "nb_field_create: bad dtype %d", (int)dt);
    if (card < 1 || card > 64) NB_FAIL(NB_EINVAL, "nb_field_create: cardinality %d", card);
    if (layout < NB_SOA || layout > NB_AOS) NB_FAIL(NB_EINVAL, "nb_field_create: bad layout %d", (int)layout);
    if (g->sparse && layout != NB_SOA && card > 1)
        NB_FAIL(NB_EUNSUPPORTED, "nb_field_create: element-sparse grids store fields as SoA");
    DeviceGuard dg(g->device);
    nb_field *f = new nb_field();
    f->g = g;
    f->dt = dt;
    f->card = card;
    f->outside = outside;
    f->esz = dt == NB_F64 ? 8 : 4;
    f->base.assign(g->nparts, nullptr);
    f->bytes.assign(g->nparts, 0);
    nb_status s = set_layout(f, layout);
    if (s != NB_OK) {
        delete f;
        return s;
    }
    if (g->sparse) {
        s = nb_sparse_field_alloc(f);
    } else {
        for (int p = 0; p < g->nparts && s == NB_OK; ++p) {
            if (!g->parts[p].local) continue;
            f->cs = nb_cstride(f, p);
            size_t bytes = (size_t)f->plane * (g->parts[p].nz() + 2) * card * f->esz;
            s = nb_field_buf_alloc(g, bytes, (void **)&f->base[p]);
            if (s != NB_OK) break;
            cudaError_t e = cudaSuccess;
            f->bytes[p] = bytes;
            if (outside == 0.0)
                e = cudaMemsetAsync(f->base[p], 0, bytes, g->cs);
            else
                s = fill_const_raw(g, f->base[p], (int64_t)(bytes / f->esz), dt, outside, g->cs);
            if (e != cudaSuccess) {
                nb_set_error("cudaMemset failed: %s", cudaGetErrorString(e));
                s = NB_ECUDA;
            }
        }
        // component stride must be uniform across partitions for the kernels'
        // per-partition arithmetic; it is per partition: store the local one
        // (all local partitions share the formula cs = ps*(nz_p+2)).
    }
    f->mapped.assign(g->nparts, 0);
    if (s == NB_OK && nb_is_peer(g)) s = nb_peer_field_map(f);  // collective
    if (s != NB_OK) {
        for (size_t p = 0; p < f->base.size(); ++p)
            if (f->base[p] && !f->mapped[p]) cudaFree(f->base[p]);
        delete f;
        return s;
    }
    g->nfields++;
    *out = f;
    return NB_OK;
}

// ---- borrowed storage (SURVEY.md §8(b) "field (borrowed)") ---------------

static nb_status required_elems(const nb_grid *g, int card, int p, int64_t *n) {
    if (p < 0 || p >= g->nparts) NB_FAIL(NB_EINVAL, "partition %d out of range", p);
    if (g->sparse)
        *n = g->sp[p].cs * card;
    else
        *n = dense_pitch(g) * g->ny * (g->parts[p].nz() + 2) * card;
    return NB_OK;
}

extern "C" nb_status nb_field_required_elems(const nb_grid *g, int32_t card, int32_t p, int64_t *n) {
    if (!g || !n || card < 1 || card > 64) NB_FAIL(NB_EINVAL, "nb_field_required_elems: bad arguments");
    return required_elems(g, card, p, n);
}

extern "C" nb_status nb_field_wrap(nb_grid *g, nb_dtype dt, int32_t card, nb_layout layout, double outside,
                                   void *const *dev_ptrs, nb_field **out) {
    if (!g || !out || !dev_ptrs) NB_FAIL(NB_EINVAL, "nb_field_wrap: NULL argument");
    *out = nullptr;
    if (layout < NB_SOA || layout > NB_AOS) NB_FAIL(NB_EINVAL, "nb_field_wrap: bad layout %d", (int)layout);
    if (dt != NB_F32 && dt != NB_F64) NB_FAIL(NB_EINVAL, "nb_field_wrap: bad dtype %d", (int)dt);
    if (card < 1 || card > 64) NB_FAIL(NB_EINVAL, "nb_field_wrap: cardinality %d", card);
    for (int i = 0; i < g->nlocal; ++i) {
        const void *ptr = dev_ptrs[i];
        if (!ptr || (uintptr_t)ptr % 16) NB_FAIL(NB_EINVAL, "nb_field_wrap: dev_ptrs[%d] is NULL or not 16-byte aligned", i);
        cudaPointerAttributes at;
        if (cudaPointerGetAttributes(&at, ptr) != cudaSuccess || at.type != cudaMemoryTypeDevice ||
            at.device != g->device) {
            cudaGetLastError();
            NB_FAIL(NB_EINVAL, "nb_field_wrap: dev_ptrs[%d] is not device memory of device %d", i, g->device);
        }
    }
    DeviceGuard dg(g->device);
    nb_field *f = new nb_field();
    f->g = g;
    f->dt = dt;
    f->card = card;
    f->outside = outside;
    f->esz = dt == NB_F64 ? 8 : 4;
    f->borrowed = true;
    f->base.assign(g->nparts, nullptr);
    f->bytes.assign(g->nparts, 0);
    f->pcs.assign(g->nparts, 0);
    f->mapped.assign(g->nparts, 0);
    nb_status s = set_layout(f, layout);
    for (int i = 0; i < g->nlocal && s == NB_OK; ++i) {
        const int p = g->first_local + i;
        int64_t n = 0;
        required_elems(g, card, p, &n);
        f->base[p] = (char *)dev_ptrs[i];
        f->bytes[p] = (size_t)n * f->esz;
        // the halo planes / segments start as outside (what nb_field_create
        // gives); own cells keep the caller's data
        if (g->sparse) {
            const NbSparsePart &sp = g->sp[p];
            f->pcs[p] = sp.cs;
            for (int c = 0; c < card && s == NB_OK; ++c) {
                char *b = f->base[p] + (size_t)c * sp.cs * f->esz;
                s = fill_const_raw(g, b, sp.hl, dt, outside, g->cs);
                if (s == NB_OK) s = fill_const_raw(g, b + (size_t)(sp.hl + sp.n) * f->esz, sp.cs - sp.hl - sp.n, dt,
                                                   outside, g->cs);
            }
        } else if (f->layout == NB_SOA) {
            const int64_t cs = nb_cstride(f, p);
            f->pcs[p] = cs;
            for (int c = 0; c < card && s == NB_OK; ++c) {
                char *b = f->base[p] + (size_t)c * cs * f->esz;
                s = fill_const_raw(g, b, f->ps, dt, outside, g->cs);
                if (s == NB_OK)
                    s = fill_const_raw(g, b + (size_t)(cs - f->ps) * f->esz, f->ps, dt, outside, g->cs);
            }
        } else {  // SOA_PLANE / AOS: a halo plane is card * plane contiguous elements
            f->pcs[p] = nb_cstride(f, p);
            const int64_t hp = f->plane * card;
            s = fill_const_raw(g, f->base[p], hp, dt, outside, g->cs);
            if (s == NB_OK) s = fill_const_raw(g, f->base[p] + (size_t)(n - hp) * f->esz, hp, dt, outside, g->cs);
        }
    }
    if (s == NB_OK) f->cs = f->pcs[g->first_local];
    if (s == NB_OK && nb_is_peer(g)) s = nb_peer_field_map(f);  // collective
    if (s != NB_OK) {
        delete f;
        return s;
    }
    g->nfields++;
    *out = f;
    return NB_OK;
}

// component stride of partition p (dense): ps * (nz_p + 2)
static inline int64_t dense_cs(const nb_field *f, int p) { return nb_cstride(f, p); }

extern "C" nb_status nb_field_destroy(nb_field *f) {
    if (!f) return NB_OK;
    DeviceGuard dg(f->g->device);
    cudaStreamSynchronize(f->g->cs);
    cudaStreamSynchronize(f->g->hs);
    if (nb_is_peer(f->g)) nb_peer_field_unmap(f);  // collective: closes the mappings, then a barrier
    for (size_t p = 0; p < f->base.size(); ++p)  // cached tensor maps over these buffers
        if (f->base[p] && p < f->bytes.size()) nb_tma_forget_range(f->base[p], f->base[p] + f->bytes[p]);
    if (!f->borrowed)
        for (size_t p = 0; p < f->base.size(); ++p)
            if (f->base[p] && !(p < f->mapped.size() && f->mapped[p]))
                nb_field_buf_release(f->g, f->base[p], p < f->bytes.size() ? f->bytes[p] : 0);
    f->g->nfields--;
    delete f;
    return NB_OK;
}

extern "C" nb_status nb_field_partition_ptr(const nb_field *f, int32_t p, void **ptr, int64_t *pitch,
                                            int64_t *pstride, int64_t *cstride) {
    if (!f || p < 0 || p >= f->g->nparts) NB_FAIL(NB_EINVAL, "nb_field_partition_ptr: bad arguments");
    if (!f->g->parts[p].local) NB_FAIL(NB_EINVAL, "partition %d is not local", p);
    if (ptr) *ptr = f->base[p];
    if (pitch) *pitch = f->pitch;
    if (pstride) *pstride = f->ps;
    if (cstride) *cstride = f->g->sparse ? f->pcs[p] : dense_cs(f, p);
    return NB_OK;
}

static size_t logical_bytes(const nb_field *f) {
    return (size_t)f->g->nx * f->g->ny * f->g->nz * f->card * f->esz;
}

// SOA_PLANE / AOS host transfers: the partition's slab of the dense logical
// view [c][z][y][x] is staged in a packed device buffer and (un)packed into
// the layout by one kernel
template <typename T, bool TO_FIELD>
__global__ void k_repack(T *field, T *packed, PGeo g, int64_t cstride, int64_t es, int card) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x, y = blockIdx.y;
    if (x >= g.nx) return;
    for (int64_t zc = blockIdx.z; zc < (int64_t)g.nzl * card; zc += gridDim.z) {
        const int zl = (int)(zc % g.nzl), c = (int)(zc / g.nzl);
        const int64_t fi = (int64_t)c * cstride + ((int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x) * es;
        const int64_t pi = (((int64_t)c * g.nzl + zl) * g.ny + y) * g.nx + x;
        if (TO_FIELD)
            field[fi] = packed[pi];
        else
            packed[pi] = field[fi];
    }
}

static nb_status dense_repack(nb_field *f, void *host, bool up) {
    nb_grid *g = f->g;
    for (int p = 0; p < g->nparts; ++p) {
        if (!g->parts[p].local) continue;
        const NbPart &q = g->parts[p];
        const size_t slab = (size_t)g->nx * g->ny * q.nz() * f->esz, logical_c = (size_t)g->nx * g->ny * g->nz * f->esz;
        void *tmp = nullptr;
        NB_CUDA(cudaMallocAsync(&tmp, slab * f->card, g->cs));
        char *h = (char *)host + (size_t)q.z0 * g->nx * g->ny * f->esz;
        PGeo geo = pgeo(f, p);
        dim3 blk(128), grd((g->nx + 127) / 128, g->ny, (unsigned)std::min<int64_t>((int64_t)geo.nzl * f->card, 65535));
        if (up)
            for (int c = 0; c < f->card; ++c)
                NB_CUDA(cudaMemcpyAsync((char *)tmp + c * slab, h + c * logical_c, slab, cudaMemcpyHostToDevice, g->cs));
        {
            LaunchScope ls(g, g->cs, "k_repack");
            if (f->dt == NB_F64 && up)
                k_repack<double, true><<<grd, blk, 0, g->cs>>>((double *)f->base[p], (double *)tmp, geo, nb_cstride(f, p),
                                                               f->es, f->card);
            else if (f->dt == NB_F64)
                k_repack<double, false><<<grd, blk, 0, g->cs>>>((double *)f->base[p], (double *)tmp, geo, nb_cstride(f, p),
                                                                f->es, f->card);
            else if (up)
                k_repack<float, true><<<grd, blk, 0, g->cs>>>((float *)f->base[p], (float *)tmp, geo, nb_cstride(f, p),
                                                              f->es, f->card);
            else
                k_repack<float, false><<<grd, blk, 0, g->cs>>>((float *)f->base[p], (float *)tmp, geo, nb_cstride(f, p),
                                                               f->es, f->card);
            NB_TRY(nb_launch_check("k_repack"));
        }
        if (!up)
            for (int c = 0; c < f->card; ++c)
                NB_CUDA(cudaMemcpyAsync(h + c * logical_c, (char *)tmp + c * slab, slab, cudaMemcpyDeviceToHost, g->cs));
        NB_CUDA(cudaFreeAsync(tmp, g->cs));
    }
    if (!up) NB_CUDA(cudaStreamSynchronize(g->cs));
    return NB_OK;
}
static nb_status dense_repack_upload(nb_field *f, const void *host) { return dense_repack(f, (void *)host, true); }
static nb_status dense_repack_download(const nb_field *f, void *host) {
    return dense_repack(const_cast<nb_field *>(f), host, false);
}

extern "C" nb_status nb_field_upload(nb_field *f, const void *host, int64_t nbytes) {
    if (!f || !host) NB_FAIL(NB_EINVAL, "nb_field_upload: NULL argument");
    if ((size_t)nbytes != logical_bytes(f))
        NB_FAIL(NB_EINVAL, "nb_field_upload: %lld bytes, expected %zu", (long long)nbytes, logical_bytes(f));
    nb_grid *g = f->g;
    DeviceGuard dg(g->device);
    if (g->sparse) return nb_sparse_upload(f, host);
    if (f->layout != NB_SOA) return dense_repack_upload(f, host);
    const char *h = (const char *)host;
    size_t row = (size_t)g->nx * f->esz, plane = row * g->ny;
    for (int p = 0; p < g->nparts; ++p) {
        if (!g->parts[p].local) continue;
        const NbPart &q = g->parts[p];
        for (int c = 0; c < f->card; ++c) {
            char *dst = f->base[p] + ((int64_t)c * dense_cs(f, p) + f->ps) * f->esz;
            const char *src = h + ((size_t)c * g->nz + q.z0) * plane;
            NB_CUDA(cudaMemcpy2DAsync(dst, f->pitch * f->esz, src, row, row, (size_t)g->ny * q.nz(),
                                      cudaMemcpyHostToDevice, g->cs));
        }
    }
    return NB_OK;
}

extern "C" nb_status nb_field_download(const nb_field *f, void *host, int64_t nbytes) {
    if (!f || !host) NB_FAIL(NB_EINVAL, "nb_field_download: NULL argument");
    if ((size_t)nbytes != logical_bytes(f))
        NB_FAIL(NB_EINVAL, "nb_field_download: %lld bytes, expected %zu", (long long)nbytes, logical_bytes(f));
    nb_grid *g = f->g;
    DeviceGuard dg(g->device);
    if (g->sparse) return nb_sparse_download(f, host);
    if (f->layout != NB_SOA) return dense_repack_download(f, host);
    char *h = (char *)host;
    size_t row = (size_t)g->nx * f->esz, plane = row * g->ny;
    for (int p = 0; p < g->nparts; ++p) {
        if (!g->parts[p].local) continue;
        const NbPart &q = g->parts[p];
        for (int c = 0; c < f->card; ++c) {
            const char *src = f->base[p] + ((int64_t)c * dense_cs(f, p) + f->ps) * f->esz;
            char *dst = h + ((size_t)c * g->nz + q.z0) * plane;
            NB_CUDA(cudaMemcpy2DAsync(dst, row, src, f->pitch * f->esz, row, (size_t)g->ny * q.nz(),
                                      cudaMemcpyDeviceToHost, g->cs));
        }
    }
    NB_CUDA(cudaStreamSynchronize(g->cs));
    return NB_OK;
}

// ---- counter-based fill: nb_gen in nb_device.cuh ----------------------------
template <typename T>
__global__ void k_fill_gen(T *base, PGeo g, int64_t cstride, int64_t es, int card, int kind, uint64_t seed,
                           double a, double b, double h) {
    int x = blockIdx.x * blockDim.x + threadIdx.x;
    int y = blockIdx.y;
    if (x >= g.nx) return;
    // (plane, component) pairs grid-strided over blockIdx.z (gridDim.z <= 65535)
    for (int64_t zc = blockIdx.z; zc < (int64_t)g.nzl * card; zc += gridDim.z) {
        int zl = (int)(zc % g.nzl);
        int c = (int)(zc / g.nzl);
        int z = g.z0 + zl;
        uint64_t gidx =
            (uint64_t)x + (uint64_t)g.nx * ((uint64_t)y + (uint64_t)g.ny * ((uint64_t)z + (uint64_t)g.NZ * c));
        double v = nb_gen(kind, seed, gidx, a, b, x, y, z, h);
        base[(int64_t)c * cstride + ((int64_t)(zl + 1) * g.ps + (int64_t)y * g.pitch + x) * es] = (T)v;
    }
}

extern "C" nb_status nb_field_fill(nb_field *f, nb_fill kind, uint64_t seed, double a, double b) {
    if (!f) NB_FAIL(NB_EINVAL, "nb_field_fill: NULL field");
    if (kind < NB_FILL_CONST || kind > NB_FILL_POISSON_RHS) NB_FAIL(NB_EINVAL, "bad fill kind");
    nb_grid *g = f->g;
    if (kind == NB_FILL_INT_UNIFORM && !(b >= a)) NB_FAIL(NB_EINVAL, "INT_UNIFORM needs b >= a");
    if (kind == NB_FILL_POISSON_RHS && !(g->nx == g->ny && g->ny == g->nz))
        NB_FAIL(NB_EUNSUPPORTED, "POISSON_RHS is defined on cubic grids");
    DeviceGuard dg(g->device);
    if (g->sparse) return nb_sparse_fill(f, kind, seed, a, b);
    double h = 1.0 / (double)(g->nx + 1);
    for (int p = 0; p < g->nparts; ++p) {
        if (!g->parts[p].local) continue;
        PGeo geo = pgeo(f, p);
        dim3 blk(128), grd((g->nx + 127) / 128, g->ny, (unsigned)std::min<int64_t>((int64_t)geo.nzl * f->card, 65535));
        LaunchScope ls(g, g->cs, "k_fill_gen");
        if (f->dt == NB_F64)
            k_fill_gen<double><<<grd, blk, 0, g->cs>>>((double *)f->base[p], geo, dense_cs(f, p), f->es, f->card,
                                                        kind, seed, a, b, h);
        else
            k_fill_gen<float><<<grd, blk, 0, g->cs>>>((float *)f->base[p], geo, dense_cs(f, p), f->es, f->card,
                                                       kind, seed, a, b, h);
        NB_TRY(nb_launch_check("k_fill_gen"));
    }
    return NB_OK;
}

// ===========================================================================
// halo update (PAPER.md L246 haloUpdate, L252 explicit transfers, L256:
// 2 transfers per component, no marshalling)
// ===========================================================================
// Components [c0, c1).  send_up: my last plane -> upper neighbour's low halo;
// send_down: my first plane -> lower neighbour's high halo.
nb_status nb_halo_exchange_planes(nb_field *f, int c0, int c1, bool send_up, bool send_down,
                                  cudaStream_t s) {
    return nb_halo_run(f, false, send_up ? c0 : 0, send_up ? c1 : 0, send_down ? c0 : 0, send_down ? c1 : 0, s);
}

nb_status nb_sparse_halo_update(nb_field *f);

// ---- split halo exchange (OCC of the sparse and FEM CG schedules) ---------
nb_status nb_halo_split_begin(nb_field *f, int c0, int c1, HaloSync &hs) {
    nb_grid *g = f->g;
    auto run = [&](cudaStream_t s, int mode) {
        return g->sparse ? nb_sparse_halo_run(f, c0, c1, c0, c1, s, mode)
                         : nb_halo_run_mode(f, false, c0, c1, c0, c1, s, mode);
    };
    if (!nb_is_peer(g) && !nb_halo_on_stream(g)) return run(g->cs, NB_HALO_GENERIC);  // one process, stream order
    if (!hs.eb) {
        NB_CUDA(cudaEventCreateWithFlags(&hs.eb, cudaEventDisableTiming));
        NB_CUDA(cudaEventCreateWithFlags(&hs.eh, cudaEventDisableTiming));
    }
    NB_CUDA(cudaEventRecord(hs.eb, g->cs));  // after the boundary-plane maps
    NB_CUDA(cudaStreamWaitEvent(g->hs, hs.eb, 0));
    NB_TRY(run(g->hs, NB_HALO_SEND));
    NB_CUDA(cudaEventRecord(hs.eh, g->hs));
    return NB_OK;
}

nb_status nb_halo_split_wait(nb_grid *g, HaloSync &hs) {
    if (!nb_is_peer(g) && !nb_halo_on_stream(g)) return NB_OK;
    if (nb_is_peer(g)) NB_TRY(nb_peer_wait(g, false, g->cs));  // the neighbours' planes are in
    NB_CUDA(cudaStreamWaitEvent(g->cs, hs.eh, 0));               // join the halo stream
    return NB_OK;
}

extern "C" nb_status nb_halo_update(nb_field *f) {
    NB_RANGE("nb_halo_update");
    if (!f) NB_FAIL(NB_EINVAL, "nb_halo_update: NULL field");
    DeviceGuard dg(f->g->device);
    if (f->g->sparse) return nb_sparse_halo_update(f);
    return nb_halo_exchange_planes(f, 0, f->card, true, true, f->g->cs);
}

// ===========================================================================
// map operations (eq. L104): y <- a*x + b*y on plane ranges, 128-bit vectors
// ===========================================================================
// The per-element arithmetic is fixed: b == 0: a*x ; b == 1: fma(a, x, y) ;
// otherwise fma(a, x, b*y).
template <typename T, int BMODE>
__device__ __forceinline__ T axpby_cell(T a, T x, T b, T y) {
    if (BMODE == 0) return a * x;
    if (BMODE == 1) return fma(a, x, y);
    return fma(a, x, b * y);
}

template <typename T, typename V, int BMODE>
__global__ void __launch_bounds__(256) k_axpby(const T *__restrict__ x, T *__restrict__ y, int64_t nvec,
                                               T a, T b) {
    constexpr int W = sizeof(V) / sizeof(T);
    const V *xv = reinterpret_cast<const V *>(x);
    V *yv = reinterpret_cast<V *>(y);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nvec;
         i += (int64_t)gridDim.x * blockDim.x) {
        V xi = __ldcs(xv + i);
        V yi;
        if (BMODE != 0) yi = __ldcs(yv + i);
        T *xs = reinterpret_cast<T *>(&xi);
        T *ys = reinterpret_cast<T *>(&yi);
        V o;
        T *os = reinterpret_cast<T *>(&o);
#pragma unroll
        for (int k = 0; k < W; ++k) os[k] = axpby_cell<T, BMODE>(a, xs[k], b, BMODE ? ys[k] : T(0));
        __stcs(yv + i, o);
    }
}

// plane ranges [zb, ze) of a view in partition p (dense)
std::vector<std::pair<int, int>> view_ranges(const nb_grid *g, int p, nb_view v) {
    const NbPart &q = g->parts[p];
    int nz = q.nz();
    int lo = q.lo >= 0 ? 1 : 0, hi = q.hi >= 0 ? 1 : 0;
    std::vector<std::pair<int, int>> r;
    if (v == NB_VIEW_STANDARD) {
        r.push_back({0, nz});
    } else if (v == NB_VIEW_INTERNAL) {
        if (nz - hi > lo) r.push_back({lo, nz - hi});
    } else {
        if (lo) r.push_back({0, 1});
        if (hi && !(lo && nz == 1)) r.push_back({nz - 1, nz});
    }
    return r;
}

static nb_status check_pair(const nb_field *x, const nb_field *y) {
    if (!x || !y) NB_FAIL(NB_EINVAL, "NULL field");
    if (x->g != y->g) NB_FAIL(NB_EMISMATCH, "fields belong to different grids");
    if (x->dt != y->dt || x->card != y->card) NB_FAIL(NB_EMISMATCH, "dtype / cardinality mismatch");
    if (x->layout != y->layout) NB_FAIL(NB_EMISMATCH, "layout mismatch");
    return NB_OK;
}

nb_status nb_sparse_axpby(double a, const nb_field *x, double b, nb_field *y, nb_view v);

template <typename T, typename V>
static nb_status launch_axpby(nb_grid *g, const T *x, T *y, int64_t n, double a, double b) {
    if (n <= 0) return NB_OK;
    constexpr int W = sizeof(V) / sizeof(T);
    int64_t nvec = n / W;  // plane ranges are multiples of 32 elements
    int blocks = (int)std::min<int64_t>((nvec + 255) / 256, 148 * 8);
    LaunchScope ls(g, g->cs, "k_axpby");
    int mode = (b == 0.0) ? 0 : (b == 1.0 ? 1 : 2);
    if (mode == 0)
        k_axpby<T, V, 0><<<blocks, 256, 0, g->cs>>>(x, y, nvec, (T)a, (T)b);
    else if (mode == 1)
        k_axpby<T, V, 1><<<blocks, 256, 0, g->cs>>>(x, y, nvec, (T)a, (T)b);
    else
        k_axpby<T, V, 2><<<blocks, 256, 0, g->cs>>>(x, y, nvec, (T)a, (T)b);
    return nb_launch_check("k_axpby");
}

extern "C" nb_status nb_axpby(double a, const nb_field *x, double b, nb_field *y, nb_view v) {
    NB_TRY(check_pair(x, y));
    if (v < NB_VIEW_STANDARD || v > NB_VIEW_BOUNDARY) NB_FAIL(NB_EINVAL, "bad view");
    nb_grid *g = x->g;
    DeviceGuard dg(g->device);
    if (g->sparse) return nb_sparse_axpby(a, x, b, y, v);
    for (int p = 0; p < g->nparts; ++p) {
        if (!g->parts[p].local) continue;
        for (auto rg : view_ranges(g, p, v)) {
            // SOA: one range per component; SOA_PLANE / AOS: the planes of
            // all components form one contiguous range
            const int nr = x->layout == NB_SOA ? x->card : 1;
            for (int c = 0; c < nr; ++c) {
                int64_t off = x->layout == NB_SOA ? (int64_t)c * dense_cs(x, p) + (int64_t)(rg.first + 1) * x->ps
                                                  : (int64_t)(rg.first + 1) * x->plane * x->card;
                int64_t n = (int64_t)(rg.second - rg.first) * x->plane * (x->layout == NB_SOA ? 1 : x->card);
                if (x->dt == NB_F64)
                    NB_TRY((launch_axpby<double, double2>(g, (const double *)x->base[p] + off,
                                                          (double *)y->base[p] + off, n, a, b)));
                else
                    NB_TRY((launch_axpby<float, float4>(g, (const float *)x->base[p] + off,
                                                        (float *)y->base[p] + off, n, a, b)));
            }
        }
    }
    return NB_OK;
}

extern "C" nb_status nb_axpy(double a, const nb_field *x, nb_field *y, nb_view v) {
    return nb_axpby(a, x, 1.0, y, v);
}

// ===========================================================================
// reduce (eq. L129): canonical tiles -> plane sums -> total
// ===========================================================================
// canonical dot tiles (the order of nb_zmarch.cuh): warp = ZR rows, per lane
// rows sequential, butterfly, then the warps of a 32 x 8 tile in order
template <typename T>
__global__ void __launch_bounds__(32 * ZW) k_dot(const T *__restrict__ x, const T *__restrict__ y, PGeo g,
                                                 int64_t cstride, int64_t es, int nchunk, double *tp, int T_tiles,
                                                 int tiles_y) {
    constexpr int ZR = ZR_STO, ZTY = ZW * ZR;
    __shared__ double sw[ZC][ZW];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int xi = blockIdx.x * DOT_TX + lane, yr = blockIdx.y * ZTY + w * ZR;
    const int c = blockIdx.z / nchunk, ch = blockIdx.z % nchunk;
    const int zs = ch * ZC, zend = min(g.nzl, zs + ZC);
    const int64_t o = (int64_t)yr * g.pitch + xi + g.ps;  // cell index; element = c * cstride + cell * es
    for (int z = zs; z < zend; ++z) {
        double col = 0.0;
#pragma unroll
        for (int j = 0; j < ZR; ++j) {
            double prod = 0.0;
            if (xi < g.nx && yr + j < g.ny) {
                const int64_t i = (int64_t)c * cstride + (o + (int64_t)z * g.ps + (int64_t)j * g.pitch) * es;
                prod = __dmul_rn((double)__ldcs(x + i), (double)__ldcs(y + i));
            }
            col = j == 0 ? prod : __dadd_rn(col, prod);
        }
        col = warp_sum_canon(col);
        if (lane == 0) sw[z - zs][w] = col;
    }
    __syncthreads();
    zm_flush<ZR>(sw, zend - zs, tp, (int64_t)c * g.NZ + g.z0 + zs, T_tiles, gridDim.x, tiles_y, blockIdx.x, blockIdx.y);
}

// ---- finalize: plane sums (one CTA per plane) + last-block total ----------

// blocks: one per plane in [p0, p1) of each component range; planes are
// indexed c*NZ + z.  If `final_planes` > 0 the last block to finish sums
// psum[0, final_planes) and applies the mode.
__global__ void __launch_bounds__(RED_THREADS) k_finalize(const double *tp, int T, double *psum,
                                                          int NZ, int z0, int zn, int card,
                                                          unsigned int *counter, int final_planes,
                                                          int mode, void *state, double *dots,
                                                          int slot) {
    __shared__ double sh[RED_THREADS];
    __shared__ int last;
    pdl_wait();  // the producing kernel's tile partials (programmatic launch)
    int b = blockIdx.x;
    int c = b / zn, z = z0 + b % zn;
    int plane = c * NZ + z;
    double s = block_tree_sum(tp + (int64_t)plane * T, T, sh);
    if (threadIdx.x == 0) psum[plane] = s;
    if (final_planes <= 0) return;
    __threadfence();
    if (threadIdx.x == 0) {
        unsigned int t = atomicAdd(counter, 1u);
        last = (t == gridDim.x - 1);
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    // canonical tree over all planes (volatile-free: psum written by other
    // blocks before their fence + atomic; read through L2); FIN_STORE_EACH:
    // the same tree over each component's planes, one total per component
    const int t = threadIdx.x;
    const int ncomp = mode == FIN_STORE_EACH ? card : 1;
    const int per = final_planes / ncomp;
    for (int cc = 0; cc < ncomp; ++cc) {
        double acc = 0.0;
        for (int i = t; i < per; i += RED_THREADS) acc = __dadd_rn(acc, __ldcg(psum + (int64_t)cc * per + i));
        sh[t] = acc;
        __syncthreads();
        for (int k = RED_THREADS / 2; k > 0; k >>= 1) {
            if (t < k) sh[t] = __dadd_rn(sh[t], sh[t + k]);
            __syncthreads();
        }
        if (t == 0) nb_apply_final(mode == FIN_STORE_EACH ? FIN_STORE : mode, sh[0], state, dots, slot + cc);
        __syncthreads();
    }
    if (t == 0) *counter = 0u;
}

__global__ void __launch_bounds__(RED_THREADS) k_final_only(const double *psum, int planes, int mode,
                                                            void *state, double *dots, int slot) {
    __shared__ double sh[RED_THREADS];
    double s = block_tree_sum(psum, planes, sh);
    if (threadIdx.x == 0) nb_apply_final(mode, s, state, dots, slot);
}

// Reduce the tile partials of `card` components (planes c*NZ + z) into the
// final value.  Single process: one launch (plane sums + last-block total).
// Multi-process: local plane sums -> NCCL all-reduce of the (disjoint,
// zero-padded) plane-sum vector -> fixed-order total on every rank.
nb_status nb_reduce_finalize(nb_grid *g, int card, int mode, void *state, int slot) {
    int planes = card * g->nz;
    cudaStream_t s = g->cs;
    bool dist = g->comm && g->comm->world > 1;
    if (!dist) {
        LaunchScope ls(g, s, "k_finalize");
        NB_CUDA(nb_launch_ex(k_finalize, dim3(planes), dim3(RED_THREADS), 0, s, true, (const double *)g->tp, g->T,
                             g->psum, (int)g->nz, 0, (int)g->nz, card, g->counter, planes, mode, state, g->dots, slot));
        return nb_launch_check("k_finalize");
    }
    if (nb_is_peer(g)) return nb_peer_reduce_finalize(g, card, mode, state, slot);
    int z0 = g->parts[g->first_local].z0, z1 = g->parts[g->first_local + g->nlocal - 1].z1;
    {
        LaunchScope ls(g, s, "k_finalize");
        k_finalize<<<card * (z1 - z0), RED_THREADS, 0, s>>>(g->tp, g->T, g->psum_send, g->nz, z0, z1 - z0,
                                                            card, g->counter, 0, mode, state, g->dots, slot);
        NB_TRY(nb_launch_check("k_finalize"));
    }
    NB_TRY(nb_nccl_allreduce_sum(g, g->psum_send, g->psum, planes, s));
    LaunchScope ls(g, s, "k_final_only");
    k_final_only<<<1, RED_THREADS, 0, s>>>(g->psum, planes, mode, state, g->dots, slot);
    return nb_launch_check("k_final_only");
}

// C1: one finalize for `iters` iterations whose tile partials sit in
// consecutive [NZ][T] slices of g->c1_tp (single process)
nb_status nb_c1_finalize_all(nb_grid *g, int iters) {
    const int planes = iters * g->nz;
    LaunchScope ls(g, g->cs, "k_finalize");
    k_finalize<<<planes, RED_THREADS, 0, g->cs>>>(g->c1_tp, g->T, g->c1_psum, g->nz, 0, g->nz, iters, g->counter,
                                                    planes, FIN_STORE_EACH, nullptr, g->dots, 0);
    return nb_launch_check("k_finalize");
}

nb_status nb_sparse_dot_partials(const nb_field *x, const nb_field *y);

// canonical tile partials of <x, y> over the planes of view v (a plane's
// partials do not depend on which launch produced them, so a split reduce —
// internal planes, then boundary planes — fills the same tiles)
nb_status nb_dot_partials_view(const nb_field *x, const nb_field *y, nb_view v) {
    nb_grid *g = x->g;
    if (g->sparse) {
        if (v != NB_VIEW_STANDARD) NB_FAIL(NB_EUNSUPPORTED, "split reduce on element-sparse grids");
        return nb_sparse_dot_partials(x, y);
    }
    for (int p = 0; p < g->nparts; ++p) {
        if (!g->parts[p].local) continue;
        for (auto rg : view_ranges(g, p, v)) {
            PGeo geo = pgeo(x, p);
            const int64_t off = (int64_t)rg.first * geo.ps * x->es * x->esz;  // planes shift, every component alike
            geo.z0 += rg.first;
            geo.nzl = rg.second - rg.first;
            int nchunk = (geo.nzl + ZC - 1) / ZC;
            dim3 blk(32 * ZW), grd(g->tiles_x, (g->ny + ZW * ZR_STO - 1) / (ZW * ZR_STO), nchunk * x->card);
            LaunchScope ls(g, g->cs, "k_dot");
            if (x->dt == NB_F64)
                k_dot<double><<<grd, blk, 0, g->cs>>>((const double *)(x->base[p] + off),
                                                       (const double *)(y->base[p] + off), geo, dense_cs(x, p), x->es, nchunk,
                                                       g->tp, g->T, g->tiles_y);
            else
                k_dot<float><<<grd, blk, 0, g->cs>>>((const float *)(x->base[p] + off),
                                                      (const float *)(y->base[p] + off), geo, dense_cs(x, p), x->es, nchunk,
                                                      g->tp, g->T, g->tiles_y);
            NB_TRY(nb_launch_check("k_dot"));
        }
    }
    return NB_OK;
}

nb_status nb_dot_partials(const nb_field *x, const nb_field *y) { return nb_dot_partials_view(x, y, NB_VIEW_STANDARD); }

extern "C" nb_status nb_dot(const nb_field *x, const nb_field *y, double *host_out) {
    NB_RANGE("nb_dot");
    NB_TRY(check_pair(x, y));
    if (!host_out) NB_FAIL(NB_EINVAL, "nb_dot: host_out is NULL");
    nb_grid *g = x->g;
    if (x->card > g->max_card) NB_FAIL(NB_EUNSUPPORTED, "nb_dot: cardinality > %d", g->max_card);
    DeviceGuard dg(g->device);
    NB_TRY(nb_dot_partials(x, y));
    NB_TRY(nb_reduce_finalize(g, x->card, FIN_STORE, nullptr, 0));
    NB_CUDA(cudaMemcpyAsync(host_out, g->dots, sizeof(double), cudaMemcpyDeviceToHost, g->cs));
    NB_CUDA(cudaStreamSynchronize(g->cs));
    return NB_OK;
}

extern "C" nb_status nb_dot_dev(const nb_field *x, const nb_field *y, double *dev_out) {
    NB_TRY(check_pair(x, y));
    if (!dev_out) NB_FAIL(NB_EINVAL, "nb_dot_dev: dev_out is NULL");
    nb_grid *g = x->g;
    if (x->card > g->max_card) NB_FAIL(NB_EUNSUPPORTED, "nb_dot_dev: cardinality > %d", g->max_card);
    DeviceGuard dg(g->device);
    NB_TRY(nb_dot_partials(x, y));
    NB_TRY(nb_reduce_finalize(g, x->card, FIN_STORE, nullptr, 0));
    NB_CUDA(cudaMemcpyAsync(dev_out, g->dots, sizeof(double), cudaMemcpyDeviceToDevice, g->cs));
    return NB_OK;
}

// ===========================================================================
// measurement
// ===========================================================================
extern "C" nb_status nb_profile_enable(nb_grid *g, int32_t enable) {
    if (!g) NB_FAIL(NB_EINVAL, "NULL grid");
    if (enable) {  // start a fresh record
        DeviceGuard dg(g->device);
        cudaStreamSynchronize(g->cs);
        for (auto &r : g->prof) {
            cudaEventDestroy(r.a);
            cudaEventDestroy(r.b);
        }
        g->prof.clear();
    }
    g->profiling = enable != 0;
    return NB_OK;
}

extern "C" nb_status nb_profile_read(nb_grid *g, const char *name, int64_t *launches, double *total_ms) {
    if (!g || !name) NB_FAIL(NB_EINVAL, "NULL argument");
    DeviceGuard dg(g->device);
    NB_CUDA(cudaStreamSynchronize(g->cs));
    NB_CUDA(cudaStreamSynchronize(g->hs));
    int64_t n = 0;
    double ms = 0.0;
    for (auto &r : g->prof) {
        if (!strstr(r.name, name)) continue;
        float t = 0.f;
        NB_CUDA(cudaEventElapsedTime(&t, r.a, r.b));
        ms += t;
        ++n;
    }
    if (launches) *launches = n;
    if (total_ms) *total_ms = ms;
    return NB_OK;
}

extern "C" nb_status nb_launch_count(const nb_grid *g, int64_t *count) {
    if (!g || !count) NB_FAIL(NB_EINVAL, "NULL argument");
    *count = g->launches;
    return NB_OK;
}
