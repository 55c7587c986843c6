// nb_peer.cu — peer-memory transport of the z-slab decomposition (one
// process per GPU, no NCCL on the data path).
//
// each partition exchanges its boundary planes with its
// two neighbours (explicit GPU-to-GPU transfers, no marshalling); L122-L131
// and L164: dot products are reduced across GPUs.  SURVEY.md §8(e) lists
// "P2P stores from the boundary kernel (fusing compute and collective)" as
// the transport; this file provides what that needs across processes:
//
//  * CUDA IPC mappings of the neighbour ranks' field partitions (so the
//    fused boundary kernels of nb_stencil.cu / nb_lbm.cu store straight
//    into the neighbour's halo plane exactly as they do between virtual
//    partitions of one process), of every rank's flag words and of every
//    rank's reduction buffer;
//  * signal / wait kernels: a system-scope release store of a device
//    counter into the consumer's flag word, an acquire spin on the
//    consumer side (bounded: a lost peer traps instead of hanging);
//  * the cross-rank dot: plane sums are stored into every rank's buffer by
//    the finalize kernel itself, whose last block raises the flags, waits
//    for all ranks and sums the planes in the canonical order — the same
//    bits as one process.
//
// Ordering argument: every halo
// consumer waits for the producer's signal of the same exchange; a producer
// writes a neighbour's halo again only after a wait that follows the
// neighbour's last read of it (ping-pong buffers in the fused LBM / CG
// schedules, an explicit "ready" round in the generic halo update), and the
// reduction buffer is double-buffered by reduction parity.
#include "nb_device.cuh"
#include "nb_internal.cuh"

#include <cuda.h>

#include <cstring>

nb_status nb_launch_check(const char *what);

// ---------------------------------------------------------------------------
// communicator
// ---------------------------------------------------------------------------
extern "C" nb_status nb_comm_create_peer(int32_t world, int32_t rank, int32_t device, nb_allgather_fn ag,
                                         void *ctx, nb_comm **out) {
    if (!out || world < 1 || world > NB_MAX_WORLD || rank < 0 || rank >= world || (world > 1 && !ag))
        NB_FAIL(NB_EINVAL, "nb_comm_create_peer: bad arguments (world %d rank %d)", world, rank);
    *out = nullptr;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess) {
        cudaGetLastError();
        ndev = 0;
    }
    if (device < 0 || device >= ndev) NB_FAIL(NB_ECUDA, "nb_comm_create_peer: device %d not available", device);
    nb_comm *c = new nb_comm();
    c->world = world;
    c->rank = rank;
    c->device = device;
    c->peer = true;
    c->ag = ag;
    c->ag_ctx = ctx;
    *out = c;
    return NB_OK;
}

extern "C" nb_status nb_comm_is_peer(const nb_comm *comm, int32_t *is_peer) {
    if (!comm || !is_peer) NB_FAIL(NB_EINVAL, "nb_comm_is_peer: NULL argument");
    *is_peer = comm->peer ? 1 : 0;
    return NB_OK;
}

static nb_status peer_allgather(nb_comm *c, const void *send, int64_t bytes, void *recv) {
    if (c->ag(c->ag_ctx, send, bytes, recv) != 0)
        NB_FAIL(NB_ENCCL, "peer transport: host allgather callback failed (%lld bytes)", (long long)bytes);
    return NB_OK;
}

nb_status nb_peer_barrier(nb_comm *c) {
    if (!c || c->world <= 1) return NB_OK;
    uint8_t one = 1;
    std::vector<uint8_t> all(c->world);
    return peer_allgather(c, &one, 1, all.data());
}

// ---------------------------------------------------------------------------
// grid: flag words, counters and the double-buffered plane-sum array
// ---------------------------------------------------------------------------
constexpr int FLAG_WORDS = 2 + NB_MAX_WORLD;
constexpr int CTR_WORDS = 8;

nb_status nb_peer_grid_setup(nb_grid *g) {
    nb_comm *c = g->comm;
    NbPeer *P = new NbPeer();
    g->peer = P;
    P->planes = g->max_card * g->nz;
    NB_CUDA(cudaMalloc(&P->flags, sizeof(uint64_t) * FLAG_WORDS));
    NB_CUDA(cudaMalloc(&P->ctr, sizeof(uint64_t) * CTR_WORDS));
    NB_CUDA(cudaMalloc(&P->psum2, sizeof(double) * 2 * P->planes));
    NB_CUDA(cudaMemset(P->flags, 0, sizeof(uint64_t) * FLAG_WORDS));
    NB_CUDA(cudaMemset(P->ctr, 0, sizeof(uint64_t) * CTR_WORDS));
    NB_CUDA(cudaMemset(P->psum2, 0, sizeof(double) * 2 * P->planes));
    NB_CUDA(cudaDeviceSynchronize());  // zeroed before any peer can signal
    cudaIpcMemHandle_t mine[2];
    NB_CUDA(cudaIpcGetMemHandle(&mine[0], P->flags));
    NB_CUDA(cudaIpcGetMemHandle(&mine[1], P->psum2));
    std::vector<cudaIpcMemHandle_t> all(2 * c->world);
    NB_TRY(peer_allgather(c, mine, sizeof(mine), all.data()));
    P->rflags.assign(c->world, nullptr);
    P->rpsum.assign(c->world, nullptr);
    for (int r = 0; r < c->world; ++r) {
        if (r == c->rank) {
            P->rflags[r] = P->flags;
            P->rpsum[r] = P->psum2;
            continue;
        }
        void *pf = nullptr, *pp = nullptr;
        NB_CUDA(cudaIpcOpenMemHandle(&pf, all[2 * r], cudaIpcMemLazyEnablePeerAccess));
        P->rflags[r] = (uint64_t *)pf;
        NB_CUDA(cudaIpcOpenMemHandle(&pp, all[2 * r + 1], cudaIpcMemLazyEnablePeerAccess));
        P->rpsum[r] = (double *)pp;
    }
    return NB_OK;
}

void nb_peer_grid_teardown(nb_grid *g) {
    NbPeer *P = g->peer;
    if (!P) return;
    for (int r = 0; r < (int)P->rflags.size(); ++r) {
        if (r == g->comm->rank) continue;
        if (P->rflags[r]) cudaIpcCloseMemHandle(P->rflags[r]);
        if (P->rpsum[r]) cudaIpcCloseMemHandle(P->rpsum[r]);
    }
    nb_peer_barrier(g->comm);  // nobody maps our buffers any more
    cudaFree(P->flags);
    cudaFree(P->ctr);
    cudaFree(P->psum2);
    delete P;
    g->peer = nullptr;
}

// ---------------------------------------------------------------------------
// fields: map the partitions adjacent to this rank's slabs (ring included,
// for periodic exchanges)
// ---------------------------------------------------------------------------
static std::vector<int> remote_neighbour_parts(const nb_grid *g) {
    std::vector<int> v;
    const int a = g->first_local, b = g->first_local + g->nlocal, n = g->nparts;
    for (int p : {a - 1, b, (a == 0 ? n - 1 : -1), (b == n ? 0 : -1)}) {
        if (p < 0 || p >= n || g->parts[p].local) continue;
        bool dup = false;
        for (int q : v) dup |= q == p;
        if (!dup) v.push_back(p);
    }
    return v;
}

// start of the cudaMalloc allocation holding p (borrowed buffers of
// nb_field_wrap may sit inside a larger, e.g. PyTorch caching-allocator, block)
typedef CUresult (*GetAddressRangeFn)(CUdeviceptr *, size_t *, CUdeviceptr);
static nb_status alloc_base(const void *p, const char **base) {
    static GetAddressRangeFn fn = nullptr;
    if (!fn) {
        void *q = nullptr;
        cudaDriverEntryPointQueryResult r;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &q, cudaEnableDefault, &r) != cudaSuccess ||
            r != cudaDriverEntryPointSuccess || !q)
            NB_FAIL(NB_ECUDA, "cuMemGetAddressRange unavailable");
        fn = (GetAddressRangeFn)q;
    }
    CUdeviceptr b = 0;
    size_t sz = 0;
    if (fn(&b, &sz, (CUdeviceptr)p) != CUDA_SUCCESS) NB_FAIL(NB_ECUDA, "cuMemGetAddressRange failed");
    *base = (const char *)b;
    return NB_OK;
}

struct IpcRec {
    cudaIpcMemHandle_t h;
    uint64_t offset;  // of the partition buffer inside the exported allocation
};

nb_status nb_peer_field_map(nb_field *f) {
    nb_grid *g = f->g;
    nb_comm *c = g->comm;
    const int k = g->nlocal;
    f->mapped.assign(g->nparts, 0);
    std::vector<IpcRec> mine(k), all((size_t)k * c->world);
    for (int i = 0; i < k; ++i) {
        const char *p = f->base[g->first_local + i], *b = p;
        if (f->borrowed) NB_TRY(alloc_base(p, &b));
        NB_CUDA(cudaIpcGetMemHandle(&mine[i].h, (void *)b));
        mine[i].offset = (uint64_t)(p - b);
    }
    NB_TRY(peer_allgather(c, mine.data(), (int64_t)sizeof(IpcRec) * k, all.data()));
    for (int p : remote_neighbour_parts(g)) {
        void *ptr = nullptr;
        NB_CUDA(cudaIpcOpenMemHandle(&ptr, all[p].h, cudaIpcMemLazyEnablePeerAccess));  // p = owner*k + index
        f->base[p] = (char *)ptr + all[p].offset;
        f->mapped[p] = 1;
        f->map_off.resize(g->nparts, 0);
        f->map_off[p] = all[p].offset;
        if (g->sparse) f->pcs[p] = g->sp[p].cs;
    }
    return NB_OK;
}

nb_status nb_peer_field_unmap(nb_field *f) {
    for (size_t p = 0; p < f->mapped.size(); ++p) {
        if (!f->mapped[p]) continue;
        cudaIpcCloseMemHandle(f->base[p] - (p < f->map_off.size() ? f->map_off[p] : 0));
        f->base[p] = nullptr;
        f->mapped[p] = 0;
    }
    return nb_peer_barrier(f->g->comm);  // no rank maps the buffers about to be freed
}

// ---------------------------------------------------------------------------
// signal / wait kernels (one thread)
// ---------------------------------------------------------------------------
struct PeerOps {
    uint64_t *ctr;
    uint64_t *sig[2];  // peer flag words to raise
    int sig_ctr[2];    // counter index per signal
    int nsig;
    const uint64_t *wait[2];  // own flag words to await
    int wait_ctr[2];
    int nwait;
    uint32_t delay_sig_ns, delay_wait_ns;  // schedule-robustness delays (nb_peer_delay)
    uint32_t jitter;
};

// ---------------------------------------------------------------------------
// Schedule-robustness delays (PAPER.md L252-L256,
// L352-L363: halo transfers and reductions are ordered by events / flags
// only, so any timing of the two sides must give the same bits).  Test
// knob, read once from the environment:
//   NB_DELAY_US     delay in microseconds (0: off)
//   NB_DELAY_WHERE  bit mask: 1 before a halo signal (producer side), 2 after
//                   a halo wait (consumer side), 4 before the reduction flags
//                   of the cross-rank dot, 8 before every batched halo copy
//                   (halo stream included)
//   NB_DELAY_RANK   the rank that is delayed (-1 or unset: every rank)
//   NB_DELAY_JITTER 1: each delay is drawn in [0, NB_DELAY_US] from the
//                   global timer instead of fixed
// ---------------------------------------------------------------------------
struct DelayCfg {
    uint32_t ns = 0, where = 0, jitter = 0;
    int rank = -1;
};
static const DelayCfg &delay_cfg() {
    static DelayCfg c = [] {
        DelayCfg d;
        if (const char *v = getenv("NB_DELAY_US")) d.ns = (uint32_t)(atof(v) * 1000.0);
        if (const char *v = getenv("NB_DELAY_WHERE")) d.where = (uint32_t)atoi(v);
        if (const char *v = getenv("NB_DELAY_RANK")) d.rank = atoi(v);
        if (const char *v = getenv("NB_DELAY_JITTER")) d.jitter = (uint32_t)atoi(v);
        return d;
    }();
    return c;
}
// delay in ns at injection point `bit` for this rank (0: none)
uint32_t nb_peer_delay(const nb_grid *g, uint32_t bit) {
    const DelayCfg &c = delay_cfg();
    if (!c.ns || !(c.where & bit)) return 0;
    const int rank = g->comm ? g->comm->rank : 0;
    return (c.rank < 0 || c.rank == rank) ? c.ns : 0;
}
uint32_t nb_peer_jitter() { return delay_cfg().jitter; }

__device__ __forceinline__ void st_release_sys(uint64_t *p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// spin until *flag >= want; a peer that never arrives (crashed rank) traps
// after 60 s instead of hanging the GPU
__device__ void peer_spin(const uint64_t *flag, uint64_t want) {
    if (ld_acquire_sys(flag) >= want) return;
    const uint64_t t0 = globaltimer_ns();
    unsigned ns = 32;
    while (ld_acquire_sys(flag) < want) {
        __nanosleep(ns);
        if (ns < 1024) ns <<= 1;
        if (globaltimer_ns() - t0 > 60ull * 1000000000ull) {
            printf("nb peer transport: timed out waiting for a peer (flag %llu < %llu)\n",
                   (unsigned long long)ld_acquire_sys(flag), (unsigned long long)want);
            __trap();
        }
    }
}

// spin for `ns` nanoseconds (jitter: a pseudo-random fraction of it)
__device__ void delay_spin(uint32_t ns, uint32_t jitter) {
    if (!ns) return;
    uint64_t t0 = globaltimer_ns();
    uint64_t d = ns;
    if (jitter) d = (t0 * 0x9E3779B97F4A7C15ull >> 40) % (uint64_t)(ns + 1);
    while (globaltimer_ns() - t0 < d) __nanosleep(256);
}

__global__ void k_delay(uint32_t ns, uint32_t jitter) {
    if (threadIdx.x == 0) delay_spin(ns, jitter);
}

nb_status nb_delay_launch(nb_grid *g, uint32_t bit, cudaStream_t s) {
    const uint32_t ns = nb_peer_delay(g, bit);
    if (!ns) return NB_OK;
    LaunchScope ls(g, s, "k_delay");
    k_delay<<<1, 32, 0, s>>>(ns, nb_peer_jitter());
    return nb_launch_check("k_delay");
}

__global__ void k_peer_ops(PeerOps o) {
    if (threadIdx.x != 0) return;
    if (o.nsig) {
        delay_spin(o.delay_sig_ns, o.jitter);
        __threadfence_system();  // this stream's earlier peer stores are performed
        for (int i = 0; i < o.nsig; ++i) {
            const uint64_t v = o.ctr[o.sig_ctr[i]] + 1;
            o.ctr[o.sig_ctr[i]] = v;
            st_release_sys(o.sig[i], v);
        }
    }
    for (int i = 0; i < o.nwait; ++i) {
        const uint64_t v = o.ctr[o.wait_ctr[i]] + 1;
        o.ctr[o.wait_ctr[i]] = v;
        peer_spin(o.wait[i], v);
    }
    if (o.nwait) {
        __threadfence_system();
        delay_spin(o.delay_wait_ns, o.jitter);
    }
}

// the ranks owning the partitions below / above this rank's slabs (-1: none)
static void neighbour_ranks(const nb_grid *g, bool per, int *lo, int *hi) {
    const int a = g->first_local, b = g->first_local + g->nlocal, n = g->nparts;
    int plo = a - 1, phi = b;
    if (plo < 0) plo = per ? n - 1 : -1;
    if (phi >= n) phi = per ? 0 : -1;
    *lo = (plo >= 0 && !g->parts[plo].local) ? nb_part_owner(g, plo) : -1;
    *hi = (phi >= 0 && !g->parts[phi].local) ? nb_part_owner(g, phi) : -1;
}

static nb_status peer_ops(nb_grid *g, bool per, bool sig, bool wait, cudaStream_t s) {
    if (!nb_is_peer(g)) return NB_OK;
    NbPeer *P = g->peer;
    int lo, hi;
    neighbour_ranks(g, per, &lo, &hi);
    PeerOps o;
    memset(&o, 0, sizeof(o));
    o.ctr = P->ctr;
    if (sig) {
        // my up-going halo lands in the upper rank's low halo: its flags[0]
        if (hi >= 0) {
            o.sig[o.nsig] = P->rflags[hi] + 0;
            o.sig_ctr[o.nsig++] = 1;
        }
        if (lo >= 0) {
            o.sig[o.nsig] = P->rflags[lo] + 1;
            o.sig_ctr[o.nsig++] = 2;
        }
    }
    if (wait) {
        if (lo >= 0) {
            o.wait[o.nwait] = P->flags + 0;
            o.wait_ctr[o.nwait++] = 3;
        }
        if (hi >= 0) {
            o.wait[o.nwait] = P->flags + 1;
            o.wait_ctr[o.nwait++] = 4;
        }
    }
    if (!o.nsig && !o.nwait) return NB_OK;
    o.delay_sig_ns = nb_peer_delay(g, 1);
    o.delay_wait_ns = nb_peer_delay(g, 2);
    o.jitter = nb_peer_jitter();
    LaunchScope ls(g, s, sig && wait ? "k_peer_round" : sig ? "k_peer_signal" : "k_peer_wait");
    k_peer_ops<<<1, 32, 0, s>>>(o);
    return nb_launch_check("k_peer_ops");
}

nb_status nb_peer_signal(nb_grid *g, bool periodic, cudaStream_t s) { return peer_ops(g, periodic, true, false, s); }
nb_status nb_peer_wait(nb_grid *g, bool periodic, cudaStream_t s) { return peer_ops(g, periodic, false, true, s); }
nb_status nb_peer_round(nb_grid *g, bool periodic, cudaStream_t s) { return peer_ops(g, periodic, true, true, s); }

// ---------------------------------------------------------------------------
// cross-rank deterministic reduction: plane sums -> every rank's psum2[par]
// -> flags -> canonical fixed-order total (identical on every rank, and
// identical to the single-process k_finalize)
// ---------------------------------------------------------------------------
struct PeerRed {
    double *psum[NB_MAX_WORLD];    // each rank's psum2
    uint64_t *rflag[NB_MAX_WORLD]; // rank r's flags[2 + me]
    const uint64_t *myflags;       // my flags[2 + r] base
    uint64_t *ctr;
    int world, rank;
    uint32_t delay_ns, jitter;  // before raising the reduction flags (nb_peer_delay bit 4)
};

__global__ void __launch_bounds__(RED_THREADS) k_finalize_peer(const double *tp, int T, int NZ, int z0, int zn,
                                                               unsigned int *counter, int planes, int mode,
                                                               void *state, double *dots, int slot, PeerRed R) {
    __shared__ double sh[RED_THREADS];
    __shared__ int last;
    const int b = blockIdx.x, t = threadIdx.x;
    const int c = b / zn, z = z0 + b % zn;
    const int plane = c * NZ + z;
    const uint64_t seq0 = R.ctr[0];
    const int par = (int)(seq0 & 1);
    // plane sum: the same fixed 256-wide tree as k_finalize
    const double s = block_tree_sum(tp + (int64_t)plane * T, T, sh);
    if (t < R.world) R.psum[t][(int64_t)par * planes + plane] = s;  // one store per rank
    __threadfence_system();
    __syncthreads();
    if (t == 0) {
        unsigned int k = atomicAdd(counter, 1u);
        last = (k == gridDim.x - 1);
    }
    __syncthreads();
    if (!last) return;
    if (t == 0) {
        __threadfence_system();
        delay_spin(R.delay_ns, R.jitter);
        const uint64_t seq = seq0 + 1;
        for (int r = 0; r < R.world; ++r)
            if (r != R.rank) st_release_sys(R.rflag[r], seq);
        for (int r = 0; r < R.world; ++r)
            if (r != R.rank) peer_spin(R.myflags + r, seq);
        __threadfence_system();
    }
    __syncthreads();
    const double *ps = R.psum[R.rank] + (int64_t)par * planes;
    double acc = 0.0;
    for (int i = t; i < planes; i += RED_THREADS) acc = __dadd_rn(acc, __ldcv(ps + i));
    sh[t] = acc;
    __syncthreads();
    for (int k = RED_THREADS / 2; k > 0; k >>= 1) {
        if (t < k) sh[t] = __dadd_rn(sh[t], sh[t + k]);
        __syncthreads();
    }
    if (t == 0) {
        *counter = 0u;
        R.ctr[0] = seq0 + 1;
        nb_apply_final(mode, sh[0], state, dots, slot);
    }
}

nb_status nb_peer_reduce_finalize(nb_grid *g, int card, int mode, void *state, int slot) {
    NbPeer *P = g->peer;
    nb_comm *c = g->comm;
    const int planes = card * g->nz;
    if (planes > P->planes) NB_FAIL(NB_EUNSUPPORTED, "peer reduction: %d planes > %d", planes, P->planes);
    const int z0 = g->parts[g->first_local].z0, z1 = g->parts[g->first_local + g->nlocal - 1].z1;
    PeerRed R;
    memset(&R, 0, sizeof(R));
    for (int r = 0; r < c->world; ++r) {
        R.psum[r] = g->peer->rpsum[r];
        R.rflag[r] = P->rflags[r] + 2 + c->rank;
    }
    R.myflags = P->flags + 2;
    R.ctr = P->ctr;
    R.world = c->world;
    R.rank = c->rank;
    R.delay_ns = nb_peer_delay(g, 4);
    R.jitter = nb_peer_jitter();
    // planes outside [z0, z1) of psum2 are filled by the other ranks; zero
    // planes of components beyond card are never read (planes = card*NZ)
    LaunchScope ls(g, g->cs, "k_finalize");
    k_finalize_peer<<<card * (z1 - z0), RED_THREADS, 0, g->cs>>>(g->tp, g->T, g->nz, z0, z1 - z0, g->counter, planes,
                                                                  mode, state, g->dots, slot, R);
    return nb_launch_check("k_finalize_peer");
}
