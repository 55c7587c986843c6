// nb_internal.cuh — shared internals of libnb (B200 / sm_100a).
//
// Everything here is product code; nothing is shared with oracle/.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <utility>
#include <string>
#include <map>
#include <vector>

#include "nb.h"

// NVTX ranges (header-only NVTX 3; free when no tool is attached): one per
// kernel enqueue (LaunchScope) and one per public operation (NB_RANGE), so
// ncu --nvtx / nsys timelines can attribute launches to library calls
#include <nvtx3/nvToolsExt.h>
struct NbRange {
    explicit NbRange(const char *name) { nvtxRangePushA(name); }
    ~NbRange() { nvtxRangePop(); }
};
#define NB_RANGE_CAT2(a, b) a##b
#define NB_RANGE_CAT(a, b) NB_RANGE_CAT2(a, b)
#define NB_RANGE(name) NbRange NB_RANGE_CAT(nb_range_, __LINE__)(name)

// ---------------------------------------------------------------------------
// error plumbing (no exception crosses the ABI)
// ---------------------------------------------------------------------------
void nb_set_error(const char *fmt, ...);

#define NB_FAIL(code, ...)            \
    do {                              \
        nb_set_error(__VA_ARGS__);    \
        return (code);                \
    } while (0)

#define NB_CUDA(call)                                                                     \
    do {                                                                                  \
        cudaError_t _e = (call);                                                          \
        if (_e != cudaSuccess)                                                            \
            NB_FAIL(NB_ECUDA, "%s failed: %s (%s:%d)", #call, cudaGetErrorString(_e),     \
                    __FILE__, __LINE__);                                                  \
    } while (0)

#define NB_TRY(call)                      \
    do {                                  \
        nb_status _s = (call);            \
        if (_s != NB_OK) return _s;       \
    } while (0)

// ---------------------------------------------------------------------------
// canonical dot tiling: every plane
// (c, z) is cut into DOT_TX x DOT_TY tiles; inside a tile each warp owns one
// x-row (lane = x), reduced by the xor-butterfly 16,8,4,2,1; the 8 warp
// values are added in increasing y; tiles of a plane and then planes are
// added by the fixed 256-wide block tree of nb_tree_sum.  Nothing depends on
// the partition count or on which kernel produced the tile value.
// ---------------------------------------------------------------------------
constexpr int DOT_TX = 32;
constexpr int DOT_TY = 8;
constexpr int RED_THREADS = 256;

// LBM lattice size
constexpr int Q19 = 19;

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int d) {
        cudaGetDevice(&prev);
        if (prev != d) cudaSetDevice(d);
    }
    ~DeviceGuard() {
        int cur = -1;
        cudaGetDevice(&cur);
        if (prev >= 0 && cur != prev) cudaSetDevice(prev);
    }
};

// largest world of the peer-memory transport (flag slots, kernel params)
constexpr int NB_MAX_WORLD = 16;

struct nb_comm {
    int world = 1, rank = 0, device = 0;
    void *nccl = nullptr;  // ncclComm_t (NCCL transport)
    // peer-memory transport (nb_comm_create_peer): host allgather used only
    // at setup (IPC handle exchange) and as the teardown barrier
    bool peer = false;
    nb_allgather_fn ag = nullptr;
    void *ag_ctx = nullptr;
};

// Per-grid state of the peer-memory transport (nb_peer.cu).  Every rank's
// flag words and reduction buffers are mapped into every other rank (CUDA
// IPC over NVLink / NVSwitch); kernels store halos and plane sums straight
// into the peer and raise a flag with a system-scope release store.
//   flags[0]      raised by the lower neighbour (its up-going halo is in)
//   flags[1]      raised by the upper neighbour (its down-going halo is in)
//   flags[2 + r]  raised by rank r (its plane sums of the current reduction)
//   ctr[0]        reductions done (parity selects the psum2 half)
//   ctr[1], [2]   halo signals sent up / down;  ctr[3], [4] halo signals
//                 awaited from below / above (device counters: CUDA-graph
//                 replay safe)
struct NbPeer {
    uint64_t *flags = nullptr;
    uint64_t *ctr = nullptr;
    double *psum2 = nullptr;  // [2][planes]
    int planes = 0;
    std::vector<uint64_t *> rflags;  // [world] each rank's flags (self: local)
    std::vector<double *> rpsum;     // [world] each rank's psum2 (self: local)
};

struct NbPart {
    int device = 0;
    int local = 1;
    int z0 = 0, z1 = 0;  // global planes [z0, z1)
    int lo = -1, hi = -1;  // neighbour partition across the low / high z face (-1: none)
    // element-sparse grids
    int64_t n_act = 0;       // active cells in the partition
    int64_t a0 = 0;          // global compact index of its first active cell
    int64_t n_lo_bnd = 0;    // active cells on the partition's first plane
    int64_t n_hi_bnd = 0;    // active cells on the partition's last plane
    int64_t halo_lo = 0;     // cells in the low halo (= previous part's last plane)
    int64_t halo_hi = 0;     // cells in the high halo (= next part's first plane)
    int nz() const { return z1 - z0; }
};

struct ProfRec {
    const char *name;
    cudaEvent_t a, b;
};

// element-sparse partition: the active cells of the
// slab in (z, y, x) order.  Field buffers hold [halo_lo | own | halo_hi]
// per component: halo_lo = the lower neighbour's last-plane cells, halo_hi =
// the upper neighbour's first-plane cells (same (y, x) order), so every halo
// transfer is one contiguous segment (no marshalling).
struct NbSparsePart {
    int64_t hl = 0, n = 0, hh = 0, cs = 0;  // halo lo / own / halo hi cells; component stride
    std::vector<int64_t> pstart;            // own-slot offset of each local plane [nz_p + 1]
    int64_t *d_pstart = nullptr;            // device copy
    int32_t *conn = nullptr;                // [6][n] buffer index of the neighbour, -1 = outside
    int32_t *conn19 = nullptr;              // D3Q19 pull sources [18][n] (lazy): -1 wall, -2 lid
    int32_t *coord = nullptr;               // [n] x | y << 16
    int max_plane = 0;                      // max active cells in one local plane
    // non-empty 256-cell dot segments, plane-major: entry = zl << 16 | seg
    int32_t *d_seg = nullptr;
    std::vector<int64_t> seg_start;         // first segment of each local plane [nz_p + 1]
    // the segments of the boundary planes facing a neighbour (OCC: one
    // launch for both), entries as d_seg (lazy)
    int32_t *d_seg_bnd = nullptr;
    int32_t *d_seg_bnd_gi = nullptr;  // their indices in the full segment table
    int64_t n_seg_bnd = -1;
    // segment-indexed 7-point neighbour table (nb_sparse.cu "segment
    // table"): d_nbr[s * 256 + t] = {-z, +z, -y | x flags, +y} offsets of the
    // segment's cell t; d_seginfo[s] = {first own cell, cells, plane << 16 |
    // index}: one dependent level before the operand gathers
    void *d_nbr = nullptr;
    void *d_seginfo = nullptr;
    int64_t n_runs = 0;
    // FEM 27-neighbourhood (lazy, nb_sparse_fem_tables): fm[j] bit
    // (ox+1) + 3(oy+1) + 9(oz+1) = that neighbour active; fb[r][j] = buffer
    // index of the first active cell among x-1 .. x+1 of row r = (oy+1) +
    // 3(oz+1), -1 if none (active cells of a row are consecutive indices)
    uint32_t *d_fm = nullptr;
    int32_t *d_fb = nullptr;
    // FEM box tables (lazy, nb_sparse_fem_box_tables): per slab row
    // (zl + 1, y), zl in [-1, nz], and 32-cell x word w: d_rm = activity
    // bits, d_ri = buffer index the word's first active cell has (or would
    // have); rw words per row.  tile_any[zl][ty][tx]: the 32 x 8 tile of
    // own plane zl holds an active node.  box_lists: (tile, z-chunk) work
    // items {tx, ty, zs, ze} per set of plane ranges
    uint32_t *d_rm = nullptr;
    int32_t *d_ri = nullptr;
    int rw = 0;
    std::vector<uint8_t> tile_any;
    // the active own nodes the box operator leaves out (element set not full
    // or gz <= 1), in plane order: 48-B records {buffer index, gz, mask, 9
    // row bases} (nb_fem.cu SpFemNode); fnode_start[zl] = first of plane zl
    void *d_fnode = nullptr;
    std::vector<int64_t> fnode_start;
    std::map<std::vector<int>, std::pair<int4 *, int64_t>> box_lists;
};

struct nb_grid {
    int nx = 0, ny = 0, nz = 0;
    int nparts = 1;
    std::vector<NbPart> parts;
    int first_local = 0, nlocal = 0;
    nb_comm *comm = nullptr;
    int device = 0;
    bool sparse = false;
    cudaStream_t cs = nullptr, hs = nullptr;
    bool own_cs = false, own_hs = false;
    // deterministic reduction scratch
    int tiles_x = 0, tiles_y = 0, T = 0;  // dot tiles per plane
    int max_card = 3;
    double *tp = nullptr;         // [max_card*nz][T] tile partials
    double *psum = nullptr;       // [max_card*nz] plane sums
    double *psum_send = nullptr;  // [max_card*nz] (multi-process)
    double *dots = nullptr;       // [NB_DOT_SLOTS] reduce results
    unsigned int *counter = nullptr;
    int nfields = 0, nsolvers = 0;
    int halo_mode = 0;  // NB_HALO_FUSED / NB_HALO_STREAM
    bool profiling = false;
    std::vector<ProfRec> prof;
    int64_t launches = 0;
    // internal scratch fields (ping-pong partners), not counted in nfields
    std::map<std::pair<int, int>, struct nb_field *> scratch;
    // CUDA graph of the last nb_map_stencil_reduce loop (key: x, y base
    // pointers, a, iterations, OCC mode) and its kernel count
    cudaGraphExec_t c1_exec = nullptr;
    const void *c1_x = nullptr, *c1_y = nullptr;
    double c1_a = 0.0;
    int c1_iters = -1, c1_occ = -1, c1_defer = -1;
    int64_t c1_launches = 0;
    // C1 tile partials / plane sums of all iterations of one call (single
    // process: one finalize per call instead of one per iteration)
    double *c1_tp = nullptr, *c1_psum = nullptr;
    // field buffer cache (single process): device buffers of destroyed
    // fields, by exact size, handed to the next field of that size instead
    // of a cudaFree / cudaMalloc pair (both synchronise and cost tens of ms
    // at GB sizes: a solver's create / destroy inside a timed region);
    // released on grid destroy or when a cudaMalloc fails
    std::multimap<size_t, void *> fcache;
    // element-sparse grids: tile partials [nz][sp_T] of the 2-phase box CG
    // (32 x 8 tiles of the bounding box, the dense canonical dot order);
    // swapped into tp / T around its kernels and finalizes (lazy)
    double *sp_tp = nullptr;
    int sp_T = 0;
    int64_t c1_cap = 0;  // doubles of c1_tp
    // element-sparse
    std::vector<NbSparsePart> sp;
    std::vector<int64_t> plane_count;  // [nz] active per global plane
    std::vector<uint8_t> host_mask;    // [z][y][x] active cells (element-sparse; lazy tables)
    int64_t n_active = 0;
    NbPeer *peer = nullptr;  // peer-memory transport (multi-process)
    // FEM: surface-node kernels concurrent with the surface-free part of the
    // streaming kernel (nb_fem.cu fem_launch): a side stream + fork/join events
    cudaStream_t fs = nullptr;
    cudaEvent_t fev[3] = {nullptr, nullptr, nullptr};
};

constexpr int NB_DOT_SLOTS = 1024;

struct nb_field {
    nb_grid *g = nullptr;
    nb_dtype dt = NB_F64;
    int card = 1;
    double outside = 0.0;
    size_t esz = 8;
    // dense layouts (include/nb.h): element (c, cell) at c*cstride + cell*es,
    // cell = (zl+1)*ps + y*pitch + x.  plane = pitch*ny cells; ps = plane
    // (SOA, AOS) or card*plane (SOA_PLANE); es = card (AOS) or 1;
    // cstride = ps*(nz_p+2) (SOA), plane (SOA_PLANE), 1 (AOS)
    nb_layout layout = NB_SOA;
    int64_t es = 1, plane = 0;
    int64_t pitch = 0, ps = 0, cs = 0;  // cells: row pitch, plane stride; cs: component stride
    std::vector<char *> base;          // per partition (local only)
    std::vector<size_t> bytes;
    std::vector<int64_t> pcs;          // per-partition component stride (elements)
    std::vector<char> mapped;          // per partition: base is a peer's buffer (CUDA IPC)
    bool borrowed = false;             // nb_field_wrap: caller-owned buffers (never freed)
    std::vector<uint64_t> map_off;     // per mapped partition: offset inside the peer's allocation
};

// component stride of partition p of a dense field (elements; see nb_field)
inline int64_t nb_cstride(const nb_field *f, int p) {
    if (f->layout == NB_SOA_PLANE) return f->plane;
    if (f->layout == NB_AOS) return 1;
    return f->ps * (f->g->parts[p].nz() + 2);
}
// fail unless f's layout is one of `mask` (1 << nb_layout)
#define NB_LAYOUTS(f, mask, what)                                                                       \
    do {                                                                                                \
        if (!((mask) & (1 << (f)->layout)))                                                             \
            NB_FAIL(NB_EUNSUPPORTED, "%s: field layout %d not supported (include/nb.h)", what, (int)(f)->layout); \
    } while (0)

// partition p's buffer of f is addressable from this process (local or mapped)
inline bool nb_reachable(const nb_field *f, int p) { return p >= 0 && f->base[p] != nullptr; }

// per-partition geometry handed to kernels (dense)
struct PGeo {
    int nx, ny, nzl;  // nzl: planes of the partition
    int z0, NZ;       // first global plane, global plane count
    int64_t pitch, ps;
};

inline PGeo pgeo(const nb_field *f, int g) {
    const NbPart &p = f->g->parts[g];
    PGeo r;
    r.nx = f->g->nx;
    r.ny = f->g->ny;
    r.nzl = p.nz();
    r.z0 = p.z0;
    r.NZ = f->g->nz;
    r.pitch = f->pitch;
    r.ps = f->ps;
    return r;
}

// pointer to plane zl (may be -1 or nzl: halo) of component c of partition g
// (SOA / SOA_PLANE: the plane's elements of that component are contiguous)
template <typename T>
inline T *plane_ptr(const nb_field *f, int g, int c, int zl) {
    return reinterpret_cast<T *>(f->base[g]) + (int64_t)c * nb_cstride(f, g) + (int64_t)(zl + 1) * f->ps * f->es;
}

// ---------------------------------------------------------------------------
// launch bookkeeping: profiling events + launch counter
// ---------------------------------------------------------------------------
struct LaunchScope {
    nb_grid *g;
    cudaStream_t s;
    const char *name;
    cudaEvent_t a = nullptr, b = nullptr;
    LaunchScope(nb_grid *g_, cudaStream_t s_, const char *n) : g(g_), s(s_), name(n) {
        nvtxRangePushA(n);
        g->launches++;
        if (g->profiling) {
            cudaEventCreate(&a);
            cudaEventCreate(&b);
            cudaEventRecord(a, s);
        }
    }
    ~LaunchScope() {
        if (g->profiling) {
            cudaEventRecord(b, s);
            g->prof.push_back({name, a, b});
        }
        nvtxRangePop();
    }
};

// Programmatic dependent launch (sm_90+): a kernel launched with
// nb_launch_ex(..., pdl = true) may start while the previous kernel of its
// stream drains; it calls pdl_wait() before touching that kernel's results
// (griddepcontrol.wait: a no-op for a normal launch), and producers call
// pdl_trigger() once their last stores are issued.  NB_NO_PDL=1 disables.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
inline bool nb_pdl_enabled() {
    return getenv("NB_NO_PDL") == nullptr;  // read per launch (graphs capture it once)
}
template <typename... KArgs, typename... Args>
inline cudaError_t nb_launch_ex(void (*k)(KArgs...), dim3 grd, dim3 blk, size_t smem, cudaStream_t s, bool pdl,
                                Args &&...args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grd;
    cfg.blockDim = blk;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = pdl && nb_pdl_enabled() ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, k, std::forward<Args>(args)...);
}

// graph instantiation flags: kernel nodes keep the priority of the stream
// they were captured on (the halo / FEM surface streams are high priority);
// NB_GRAPH_PRIO=0 instantiates without node priorities
inline unsigned long long nb_graph_flags() {
    const char *v = getenv("NB_GRAPH_PRIO");
    return (v && atoi(v) == 0) ? 0ull : (unsigned long long)cudaGraphInstantiateFlagUseNodePriority;
}

// kernels / helpers implemented in the .cu files
nb_status nb_launch_check(const char *what);
nb_status nb_reduce_finalize(nb_grid *g, int planes, int mode, void *state, int slot);

// finalize modes
enum {
    FIN_STORE = 0,    // dots[slot] = total
    FIN_CG_INIT = 1,  // rr = rr0 = total
    FIN_CG_PQ = 2,    // alpha = rr / total
    FIN_CG_RR = 3,    // beta = total / rr ...
    FIN_STORE_EACH = 4,  // dots[slot + c] = total of component c (card components)
};

struct CgScal {
    double rr, rr0, alpha, alpha_prev, beta, pq, rtol2;
    int32_t iters, status, pending, pad;
};

// apply a reduction's total: store it, or advance the CG scalars (the
// convergence gate of SURVEY.md §8(c) c5 lives here, on the device)
__device__ __forceinline__ void nb_apply_final(int mode, double total, void *state, double *dots, int slot) {
    if (mode == FIN_STORE) {
        dots[slot] = total;
        return;
    }
    CgScal *s = (CgScal *)state;
    if (mode == FIN_CG_INIT) {
        s->rr = total;
        s->rr0 = total;
        s->status = (total == 0.0) ? 2 : 0;
        s->alpha = 0.0;
        s->alpha_prev = 0.0;
        s->beta = 0.0;
        s->pending = 0;
        s->iters = 0;
        return;
    }
    if (s->status != 0) return;
    if (mode == FIN_CG_PQ) {
        s->pq = total;
        s->pending = 0;  // phase A applied the deferred x update
        if (!(total > 0.0))
            s->status = 3;
        else
            s->alpha = s->rr / total;
    } else if (mode == FIN_CG_RR) {
        s->beta = total / s->rr;
        s->rr = total;
        s->alpha_prev = s->alpha;
        s->pending = 1;
        s->iters += 1;
        if (total == 0.0)
            s->status = 2;
        else if (s->rtol2 > 0.0 && total <= s->rtol2 * s->rr0)
            s->status = 1;
    }
}

nb_status nb_grid_alloc_common(nb_grid *g);
nb_status nb_grid_setup_parts(nb_grid *g, const int32_t *zb, int32_t nparts, const int32_t *device_ids,
                              nb_comm *comm);
// cached internal field of the grid (slot distinguishes several of one kind)
nb_status nb_grid_scratch(nb_grid *g, nb_dtype dt, int card, int slot, nb_field **out);

// Batched plane copies (one launch for all device-local / peer-mapped halo
// planes of an exchange): up to MAX (dst, src, bytes) descriptors passed by
// value; blocks are dealt to descriptors by a prefix of block counts.
// 16-byte vectors when every address and size allows it, else 4-byte words.
struct CopyBatch {
    static constexpr int MAX = 48;
    static constexpr int CHUNK = 256 * 4;  // vectors per block
    void *dst[MAX];
    const void *src[MAX];
    uint64_t words[MAX];     // number of 16-byte (vec) or 4-byte words
    uint32_t bstart[MAX + 1];
    uint64_t vec;            // bit i: descriptor i uses 16-byte words
    int n = 0;
    static_assert(MAX <= 64, "CopyBatch::vec holds one bit per descriptor");
    CopyBatch() : vec(0) { bstart[0] = 0; }
    void add(void *d, const void *s_, size_t bytes) {
        bool v = ((uintptr_t)d % 16 == 0) && ((uintptr_t)s_ % 16 == 0) && (bytes % 16 == 0);
        dst[n] = d;
        src[n] = s_;
        words[n] = v ? bytes / 16 : bytes / 4;
        if (v) vec |= 1ull << n;
        bstart[n + 1] = bstart[n] + (uint32_t)((words[n] + CHUNK - 1) / CHUNK);
        ++n;
    }
};
nb_status nb_launch_copy_batch(nb_grid *g, const CopyBatch &cb, cudaStream_t s);
// drop cached TMA tensor maps whose base address lies in [lo, hi) (nb_tma.cu)
void nb_tma_forget_range(const void *lo, const void *hi);

// halo helpers (nb_api.cu)
nb_status nb_halo_exchange_planes(nb_field *f, int c0, int c1, bool send_up, bool send_down,
                                  cudaStream_t s);
nb_status nb_halo_run(nb_field *f, bool periodic, int c0u, int c1u, int c0d, int c1d, cudaStream_t s);
// halo modes: GENERIC = with the peer transport a "ready" round before and a
// "done" round after the copies; SEND = the copies and a signal only (the
// consumer waits; used where a reduction already orders the previous read
// before the next write)
enum { NB_HALO_GENERIC = 0, NB_HALO_SEND = 1 };
nb_status nb_halo_run_mode(nb_field *f, bool periodic, int c0u, int c1u, int c0d, int c1d, cudaStream_t s,
                           int mode);
nb_status nb_sparse_halo_run(nb_field *f, int c0u, int c1u, int c0d, int c1d, cudaStream_t s, int mode);
// element-sparse FEM (nb_sparse.cu tables, nb_fem.cu operator)
nb_status nb_sparse_fem_tables(nb_grid *g, bool with_bases);  // fm; fb (gather pass) if with_bases
// one pass of the sparse FEM operator over segment list entries [s0, s0+n) of
// `list` (gidx: their global segment indices, NULL = s0 + q) of partition p.
// kind: 0 = y = K u, 1 = q = K u with <u, q>, 2 = y = b - K u with <y, y>
nb_status nb_sparse_fem_pass(nb_grid *g, int p, int kind, const int32_t *list, const int32_t *gidx, int64_t s0,
                             int64_t n, const double *u, const double *b, double *y, const CgScal *sc);
// the same operator from shared-memory boxes (k_sp_fem_box): the output
// planes of the local plane ranges {zb0, ze0, zb1, ze1, ...} of partition p.
// kind: 0 = y = K u, 2 = y = b - K u (no dot: nb_sparse_fem_dot); sc != NULL
// makes it a no-op once the solver stopped.  Same values as the gather pass.
bool nb_sparse_fem_boxed();  // the box operator is the default (NB_SPF_GATHER=1: the gather pass)
nb_status nb_sparse_fem_box_tables(nb_grid *g);
nb_status nb_sparse_fem_box_list(nb_grid *g, int p, const std::vector<int> &ranges, int zc, const int4 **items,
                                 int64_t *n, bool all = false, int th = 8);
nb_status nb_sparse_tile_tp(nb_grid *g);
// field buffers through the grid's cache (nb_api.cu)
nb_status nb_field_buf_alloc(nb_grid *g, size_t bytes, void **out);
void nb_field_buf_release(nb_grid *g, void *buf, size_t bytes);
void nb_field_cache_clear(nb_grid *g);
// the grid's tile partial buffer (sp_tp, sp_T) in place of the segment
// partials for the box kernels' dots and the finalize that reads them
struct SpTpSwap {
    nb_grid *g;
    double *tp;
    int T;
    explicit SpTpSwap(nb_grid *g_) : g(g_), tp(g_->tp), T(g_->T) {
        g->tp = g->sp_tp;
        g->T = g->sp_T;
    }
    ~SpTpSwap() {
        g->tp = tp;
        g->T = T;
    }
};
// kind 3 (sparse FEM CG phase A): p_new = r + beta p_old, deferred x, q = K
// p_new in one pass (the CG's buffers below; p ping-pongs by parity)
struct SpFemCgA {
    const double *r, *po;
    double *pn, *x;
};
nb_status nb_sparse_fem_box(nb_grid *g, int p, int kind, const std::vector<int> &ranges, const double *u,
                            const double *b, double *y, const CgScal *sc, const SpFemCgA *cga = nullptr);
// p_new on the boundary planes facing a neighbour (before their halo is sent)
nb_status nb_sparse_pmap(nb_grid *g, int p, int card, const double *po, const double *r, double *pn,
                         const CgScal *sc);
// per-segment partials of <a, b> over the 3 components of partition p (the
// gather pass's dot, bit for bit), all segments
nb_status nb_sparse_fem_dot(nb_grid *g, int p, const double *a, const double *b, const CgScal *sc);
// the box operator over local planes: which = 0 all, 1 the interior (planes
// whose neighbours are own planes), 2 the boundary planes facing a neighbour
nb_status nb_sparse_fem_box_ranges(nb_grid *g, int p, int which, const double *u, const double *b, double *y,
                                   const CgScal *sc, int kind, const SpFemCgA *cga);
nb_status nb_sparse_fem_box_prepare(nb_grid *g);  // tables + every list (call outside graph capture)
nb_status nb_nccl_allreduce_sum(nb_grid *g, const double *send, double *recv, size_t n,
                                cudaStream_t s);
nb_status nb_nccl_group(nb_grid *g, bool start);
nb_status nb_nccl_send(nb_grid *g, const void *buf, size_t bytes, int peer, cudaStream_t s);
nb_status nb_nccl_recv(nb_grid *g, void *buf, size_t bytes, int peer, cudaStream_t s);

int nb_part_owner(const nb_grid *g, int part);
// y = L(x) or y = -L(x) on a view (nb_stencil.cu); the D3Q19 step of fin
// into fout on a view without fused halo stores (nb_lbm.cu): Skeleton nodes
nb_status nb_stencil7(const nb_field *x, nb_field *y, nb_view v, bool neg);
nb_status nb_lbm_view(nb_field *fin, nb_field *fout, const nb_lbm_params *prm, nb_view v);
std::vector<std::pair<int, int>> view_ranges(const nb_grid *g, int p, nb_view v);
// multi-process with the peer-memory transport
inline bool nb_is_peer(const nb_grid *g) { return g->comm && g->comm->world > 1 && g->comm->peer; }
// multi-process with the NCCL transport
inline bool nb_is_nccl(const nb_grid *g) { return g->comm && g->comm->world > 1 && !g->comm->peer; }
// halos travel on the halo stream (NCCL transport, or NB_HALO_STREAM);
// otherwise the boundary kernels store them straight into the neighbour
// (same process, or a peer's buffer mapped through CUDA IPC)
inline bool nb_halo_on_stream(const nb_grid *g) { return nb_is_nccl(g) || g->halo_mode == NB_HALO_STREAM; }

// peer-memory transport (nb_peer.cu)
nb_status nb_peer_grid_setup(nb_grid *g);
void nb_peer_grid_teardown(nb_grid *g);
nb_status nb_peer_field_map(struct nb_field *f);
nb_status nb_peer_field_unmap(struct nb_field *f);
// halo signal to / wait for the neighbouring ranks (periodic: ring too)
nb_status nb_peer_signal(nb_grid *g, bool periodic, cudaStream_t s);
nb_status nb_peer_wait(nb_grid *g, bool periodic, cudaStream_t s);
// signal + wait in one launch
nb_status nb_peer_round(nb_grid *g, bool periodic, cudaStream_t s);
nb_status nb_peer_barrier(nb_comm *c);
nb_status nb_peer_reduce_finalize(nb_grid *g, int card, int mode, void *state, int slot);
// schedule-robustness test knob (NB_DELAY_* environment, nb_peer.cu): the
// delay in ns at injection point `bit` for this rank, and a spin kernel
uint32_t nb_peer_delay(const nb_grid *g, uint32_t bit);
nb_status nb_delay_launch(nb_grid *g, uint32_t bit, cudaStream_t s);

// halo overlap events of a schedule (multi-process)
struct HaloSync {
    cudaEvent_t eb = nullptr, eh = nullptr;
};
// OCC split of a halo exchange of components [c0, c1) (sparse and FEM CG):
// begin after the boundary-plane maps (the transfer runs on the halo stream
// with the peer / NCCL transport or NB_HALO_STREAM, in stream order
// otherwise); wait before the boundary-plane stencils
nb_status nb_halo_split_begin(nb_field *f, int c0, int c1, HaloSync &hs);
nb_status nb_halo_split_wait(nb_grid *g, HaloSync &hs);

#include <map>
struct nb_cg {
    nb_grid *g = nullptr;
    nb_field *x = nullptr;
    const nb_field *b = nullptr;
    nb_field *r = nullptr, *p[2] = {nullptr, nullptr}, *q = nullptr;
    CgScal *sc = nullptr;
    nb_cg_params prm{};
    int64_t k = 0;  // iterations enqueued
    std::map<std::pair<int, int>, std::pair<cudaGraphExec_t, int64_t>> graphs;  // (count, parity) -> graph, kernels
    HaloSync hs;
    bool finished = false;
    // sparse CG with the fused phase A (the 2-phase box CG, or the FEM
    // NB_SPF_FUSED path): p ping-pongs by iteration parity (as in the dense
    // CG), so the final flush picks p by sc->iters
    bool pingpong = false;
    bool sp_box = false;  // sparse 7-point CG on the 2-phase box schedule
};

