/*
 * nb.h — C ABI of the B200-native Neon map-stencil hot path
 * (Meneghin, Mahmoud, Jayaraman, Morris, "Neon: A Multi-GPU Programming
 * Model for Grid-based Computations", IPDPS 2022 — /root/reference/PAPER.md,
 * cited as L<line>).
 *
 * Library: paper_conf_ipps_meneghinmjm22_b200/libnb.so (sm_100a).
 *
 * Conventions:
 *  - Every function returns nb_status: NB_OK (0) or an error code; no C++
 *    exception crosses the ABI.  nb_last_error() returns a thread-local
 *    message for the last failing call on the calling thread.
 *  - Errors from asynchronous GPU work surface at the next synchronising
 *    call (nb_sync, nb_dot, nb_field_download, nb_cg_finish, ...).
 *  - Handles are opaque and caller-owned; *_destroy(NULL) is a no-op.
 *    A grid must outlive its fields and solvers (NB_ESTATE otherwise).
 *  - Host pointers are borrowed for the duration of the call only.
 *  - Operations are stream-ordered on the grid's compute stream and return
 *    immediately, except where "synchronises" is stated.
 *  - Dense host logical view ("Host Logical View"):
 *    element (c, x, y, z) of a field is host[x + Nx*(y + Ny*(z + Nz*c))].
 *  - A grid is driven by one host thread at a time.
 *  - There is no CPU fallback: without a CUDA device every call that needs
 *    one fails with NB_ECUDA.
 */
#ifndef NB_H
#define NB_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t nb_status;
#define NB_OK 0
#define NB_EINVAL 1        /* bad argument (NULL handle, size, range, ...)        */
#define NB_ENOMEM 2        /* device or host allocation failed                    */
#define NB_ECUDA 3         /* CUDA runtime error (incl. no device)                */
#define NB_ENCCL 4         /* NCCL missing or failed                              */
#define NB_EMISMATCH 5     /* fields of different grids / dtype / cardinality     */
#define NB_EUNSUPPORTED 6  /* valid request this build does not support           */
#define NB_ESTATE 7        /* object in the wrong state (live fields, reuse, ...) */

typedef enum { NB_F32 = 0, NB_F64 = 1 } nb_dtype;

/* Data views: Internal cells need only partition-local data;
 * Boundary cells read halo data received from a neighbouring partition;
 * Standard = Internal U Boundary.  With radius-1 stencils and z-slab
 * partitions the Boundary view is the first and/or last plane of a slab that
 * faces another partition; global domain faces are Internal. */
typedef enum { NB_VIEW_STANDARD = 0, NB_VIEW_INTERNAL = 1, NB_VIEW_BOUNDARY = 2 } nb_view;

/* Overlap of computation and communication (Fig. 1,
 * L293-L315): NONE = global barrier before the halo update; STANDARD = split
 * the stencil into internal/boundary, overlap the halo with the internal part;
 * EXTENDED = also split the preceding map and send the halo right after the
 * boundary map; TWO_WAY = EXTENDED + split the following reduce. */
typedef enum { NB_OCC_NONE = 0, NB_OCC_STANDARD = 1, NB_OCC_EXTENDED = 2, NB_OCC_TWO_WAY = 3 } nb_occ;

/* Synthetic, partition-independent initialisation (DESIGN.md "Input
 * recipe"): CONST = a; UNIFORM = a + (b-a)*u, u = (h>>11)*2^-53;
 * INT_UNIFORM = a + (h mod (b-a+1)) (a, b integers); POISSON_RHS = h^2 f of
 * the manufactured solution g(x)g(y)g(z), g(t) = t(1-t) (cubic grids only);
 * h = splitmix64(seed*0x9E3779B97F4A7C15 + gidx + 1) with
 * gidx = x + Nx*(y + Ny*(z + Nz*c)). */
typedef enum {
    NB_FILL_CONST = 0,
    NB_FILL_UNIFORM = 1,
    NB_FILL_INT_UNIFORM = 2,
    NB_FILL_POISSON_RHS = 3
} nb_fill;

typedef struct nb_comm nb_comm;
typedef struct nb_grid nb_grid;
typedef struct nb_field nb_field;
typedef struct nb_cg nb_cg;

/* ---- library ---------------------------------------------------------- */
const char *nb_version(void);
const char *nb_last_error(void);
/* number of CUDA devices visible (0 on a CPU-only host; never fails) */
int32_t nb_device_count(void);

/* ---- communicator (one process per GPU; PAPER.md L238 multi-GPU streams,
 * L252-L256 explicit GPU-GPU transfers).  Built on NCCL, loaded at run time
 * (dlopen libnccl.so.2); NB_ENCCL if it cannot be loaded. --------------- */
/* out: 128 opaque bytes to broadcast from rank 0 to every rank */
nb_status nb_comm_unique_id(uint8_t out[128]);
/* world >= 1 processes; rank in [0, world); device = the CUDA device this
 * process drives.  Collective over all ranks. */
nb_status nb_comm_create(int32_t world, int32_t rank, const uint8_t id[128], int32_t device,
                         nb_comm **out);
nb_status nb_comm_destroy(nb_comm *comm);

/* Peer-memory transport (PAPER.md L252-L256 explicit GPU-to-GPU transfers,
 * SURVEY.md §8(e) "P2P stores from the boundary kernel"): no NCCL on the
 * data path.  Every field partition adjacent to this rank's slabs, and every
 * rank's reduction buffer and flag words, are mapped into this process with
 * CUDA IPC; boundary kernels store their halo planes straight into the
 * neighbour's halo (over NVLink / NVSwitch, or locally when several
 * processes share one GPU), plane sums of a reduction are stored into every
 * rank, and completion is a system-scope release store of a counter that
 * the consumer's kernel acquires.  Ordering is stream order + these flags.
 *
 * ag(ctx, send, bytes, recv): host allgather used ONLY during setup and
 * teardown (IPC handle exchange, barrier): every rank passes `bytes` bytes,
 * recv receives world*bytes bytes ordered by rank; return 0 on success.
 * It is called from inside nb_grid_create_*, nb_grid_destroy,
 * nb_field_create and nb_field_destroy, which therefore become collective:
 * every rank makes the same calls in the same order.  world <= 16.
 * Comm and callback must outlive every grid built on them. */
typedef int32_t (*nb_allgather_fn)(void *ctx, const void *send, int64_t bytes, void *recv);
nb_status nb_comm_create_peer(int32_t world, int32_t rank, int32_t device, nb_allgather_fn ag, void *ctx,
                              nb_comm **out);
/* 1 if comm uses the peer-memory transport, 0 if NCCL */
nb_status nb_comm_is_peer(const nb_comm *comm, int32_t *is_peer);

/* ---- grid (PAPER.md L81-L88 Domain, L244 Grid, L256 1-D decomposition) -- */
/* Pure host logic (no GPU needed): the z-slab partition of a1 — partition g
 * owns planes [z_begin[g], z_begin[g+1]); the first (nz mod nparts)
 * partitions get one extra plane.  z_begin has nparts+1 entries.
 * NB_EINVAL if nparts < 1 or any slab would be empty. */
nb_status nb_partition_plan(int32_t nz, int32_t nparts, int32_t *z_begin);
/* Pure host logic: active-count balanced plane cuts for an element-sparse
 * grid: counts[z] active cells per plane; cut g+1 is the
 * first plane whose prefix count reaches (g+1)*total/nparts, with every slab
 * non-empty. */
nb_status nb_partition_plan_weighted(int32_t nz, const int64_t *counts, int32_t nparts,
                                     int32_t *z_begin);

/* One halo message of the z-slab decomposition (each
 * partition talks to its two neighbours; 2 transfers per component, no
 * marshalling). */
typedef struct {
    int32_t src_part, dst_part;  /* global partition ids                          */
    int32_t src_rank, dst_rank;  /* owning processes (equal: a device copy)       */
    int32_t src_plane;           /* local plane of src sent (0 or nz_src-1)        */
    int32_t dst_plane;           /* halo plane of dst written (-1 or nz_dst)       */
    int32_t up;                  /* 1: src's top plane -> dst's low halo; 0: down */
} nb_halo_msg;
/* Pure host logic: the halo messages of an nparts-slab decomposition of nz
 * planes owned by `world` processes (partition p on rank p/(nparts/world)),
 * restricted to those `rank` sends or receives (rank = -1: all), in the
 * canonical order every rank posts them in (so point-to-point sends and
 * receives between two ranks match in order): neighbour pairs (p, p+1) in
 * increasing p — with periodic != 0 also the ring pair (nparts-1, 0) — and
 * within a pair the up message before the down message.  count receives the
 * number of messages; out may be NULL to query it; NB_EINVAL if cap is too
 * small. */
nb_status nb_halo_plan(int32_t nz, int32_t nparts, int32_t world, int32_t rank, int32_t periodic,
                       nb_halo_msg *out, int32_t cap, int32_t *count);

/* Dense grid of dims = {Nx, Ny, Nz} cells split into nparts z-slabs.
 * comm == NULL: every partition lives in this process; device_ids[nparts]
 *   gives each partition's device and must name ONE device (virtual
 *   partitions: several partitions on one GPU — the multi-GPU schedule,
 *   halo copies and reductions run unchanged, which is what the
 *   partition-invariance tests use).
 * comm != NULL: nparts must be a multiple of the world size; this rank owns
 *   partitions [rank*k, (rank+1)*k), k = nparts/world, all on comm's device
 *   (device_ids may be NULL).
 * NB_EUNSUPPORTED if nparts > 1 and a slab has fewer than 2 planes. */
nb_status nb_grid_create_dense(const int32_t dims[3], int32_t nparts, const int32_t *device_ids,
                               nb_comm *comm, nb_grid **out);
/* Element-sparse grid: active[z][y][x] (0/1, Nx*Ny*Nz
 * bytes, copied) selects the stored cells; the connectivity table is built
 * on the device.  Cuts balance the active count (nb_partition_plan_weighted). */
nb_status nb_grid_create_sparse(const int32_t dims[3], const uint8_t *active, int32_t nparts,
                                const int32_t *device_ids, nb_comm *comm, nb_grid **out);
nb_status nb_grid_destroy(nb_grid *grid);

typedef struct {
    int32_t device;      /* CUDA device of the partition                         */
    int32_t local;       /* 1 if owned by this process                           */
    int32_t z_begin;     /* first global plane                                   */
    int32_t z_end;       /* one past the last global plane                       */
    int64_t n_cells;     /* active cells in the partition                        */
    int64_t n_bnd_lo;    /* cells of the Boundary view on the low-z side         */
    int64_t n_bnd_hi;    /* cells of the Boundary view on the high-z side        */
    int64_t n_internal;  /* cells of the Internal view                           */
} nb_part_info;
nb_status nb_grid_num_partitions(const nb_grid *grid, int32_t *nparts);
nb_status nb_grid_partition_info(const nb_grid *grid, int32_t g, nb_part_info *out);
/* Use caller streams (e.g. torch.cuda.Stream.cuda_stream) instead of the
 * library's own.  Either may be NULL to keep the current one. */
nb_status nb_grid_set_streams(nb_grid *grid, void *compute_stream, void *halo_stream);
nb_status nb_grid_get_stream(const nb_grid *grid, void **compute_stream);
/* Halo transport for partitions of this process: NB_HALO_FUSED (default)
 * stores boundary-plane outputs straight into the neighbour's halo from the
 * producing kernel; NB_HALO_STREAM issues them as device copies on the halo
 * stream, ordered by events and overlapped with the interior kernels (the
 * cross-process path always uses the halo stream, with NCCL). */
#define NB_HALO_FUSED 0
#define NB_HALO_STREAM 1
nb_status nb_grid_set_halo_mode(nb_grid *grid, int32_t mode);
/* synchronises: waits for all work of the grid, reports async errors */
nb_status nb_sync(nb_grid *grid);
/* Waits for the grid's streams and frees the field buffer cache (the device
 * buffers of destroyed fields, see nb_field_destroy); *freed_bytes (may be
 * NULL) receives their total size. */
nb_status nb_grid_trim(nb_grid *grid, int64_t *freed_bytes);

/* ---- fields (PAPER.md L58-L63 newField<T>(cardinality, outsideDomainValue),
 * L246 Field, L248 "SoA or AoS organizations without impacting the
 * application code", L252 halo regions) -----------------------------------
 * Device layouts per dense partition (x-rows padded to a 32-element pitch,
 * one halo plane below and above the slab, zl = -1 .. nz_g):
 *   NB_SOA        [c][zl][y][x]  a component's planes contiguous; a halo
 *                 exchange is one transfer per component and direction
 *                 (2 x C per partition, L256)
 *   NB_SOA_PLANE  [zl][c][y][x]  the components of a plane contiguous: any
 *                 component range of a plane is ONE transfer (L256 "2")
 *   NB_AOS        [zl][y][x][c]  the components of a cell contiguous; a
 *                 halo plane moves whole (all components, one transfer)
 * Element (c, x, y, zl) sits at c*cstride + ((zl+1)*pstride + y*pitch + x)*estride
 * (nb_field_partition_ptr; estride = C for AOS, else 1).  Cardinality 1:
 * the three layouts coincide (reported as NB_SOA).  Halo planes facing the
 * global domain boundary hold outside_value (the value read for out-of-domain
 * neighbours).  Maps, dots, halo updates, upload / download / fill, the
 * 7-point stencil and the D3Q19 twoPop step take every layout; the FEM
 * operator takes SOA and SOA_PLANE; other operations (AA pattern, D2Q9,
 * element-sparse grids) take SOA only and return NB_EUNSUPPORTED otherwise.
 * Sparse grids: [c][-halo_lo .. n_g + halo_hi) over the partition's active
 *   cells in (z, y, x) order. */
typedef enum { NB_SOA = 0, NB_SOA_PLANE = 1, NB_AOS = 2 } nb_layout;
nb_status nb_field_create(nb_grid *grid, nb_dtype dtype, int32_t cardinality, nb_layout layout,
                          double outside_value, nb_field **out);
/* Waits for the grid's streams.  In one process the field's device buffers
 * go to the grid's cache and are handed to the next field of the same size
 * (no cudaFree / cudaMalloc pair); the cache is freed by nb_grid_destroy and
 * whenever a later allocation fails (NB_NO_FIELD_CACHE=1 frees at once).
 * Borrowed buffers (nb_field_wrap) stay the caller's. */
nb_status nb_field_destroy(nb_field *field);
/* Borrowed storage (SURVEY.md §8(b) "field (borrowed)": PyTorch owns the
 * memory).  Pure host logic: the number of elements partition g of a field
 * of `cardinality` components occupies in the layout above (dense:
 * pitch*Ny*(nz_g+2)*card; sparse: (halo_lo+n_g+halo_hi, padded)*card). */
nb_status nb_field_required_elems(const nb_grid *grid, int32_t cardinality, int32_t g, int64_t *n);
/* A field over caller-owned device buffers: dev_ptrs[i] backs the i-th
 * partition owned by this process (partitions in increasing order), each at
 * least nb_field_required_elems elements of dtype, 16-byte aligned, on the
 * grid's device.  The call writes outside_value into the halo planes /
 * segments (stream-ordered) and leaves the own cells as they are; the
 * library never frees the buffers — the caller keeps them alive until
 * nb_field_destroy.  NB_EINVAL for NULL, misaligned or non-device pointers.
 * With the peer transport the call is collective, like nb_field_create. */
nb_status nb_field_wrap(nb_grid *grid, nb_dtype dtype, int32_t cardinality, nb_layout layout,
                        double outside_value, void *const *dev_ptrs, nb_field **out);
/* the field's layout (cardinality 1: NB_SOA) */
nb_status nb_field_layout(const nb_field *field, nb_layout *layout);
/* host: dense logical view, nbytes = Nx*Ny*Nz*card*sizeof(dtype); inactive
 * cells of sparse grids are ignored on upload and read back as outside.
 * Upload is stream-ordered (host buffer must stay valid until nb_sync);
 * download synchronises. */
nb_status nb_field_upload(nb_field *field, const void *host, int64_t nbytes);
nb_status nb_field_download(const nb_field *field, void *host, int64_t nbytes);
nb_status nb_field_fill(nb_field *field, nb_fill kind, uint64_t seed, double a, double b);
/* haloUpdate: copy every partition's boundary planes into
 * its neighbours' halo planes (2 transfers per component, L256). */
nb_status nb_halo_update(nb_field *field);
/* device pointer of partition g's buffer (element (c, x, y, zl) at
 * ptr + c*cstride + ((zl+1)*pstride + y*pitch + x)*estride, in elements;
 * estride: see the layouts above) */
nb_status nb_field_partition_ptr(const nb_field *field, int32_t g, void **ptr, int64_t *pitch,
                                 int64_t *pstride, int64_t *cstride);

/* ---- map, stencil, reduce (eqs.) ---- */
/* y <- a*x + y on the view (one fused multiply-add per element) */
nb_status nb_axpy(double a, const nb_field *x, nb_field *y, nb_view view);
/* y <- a*x + b*y; b == 0 writes a*x without reading y (copy/scale) */
nb_status nb_axpby(double a, const nb_field *x, double b, nb_field *y, nb_view view);
/* y <- L(x), L(x)_i = sum of the 6 face neighbours - 6 x_i (Listing 2,
 * L145-L152), out-of-domain neighbours read x's outside_value.  Reads x's
 * halo planes as they are: call nb_halo_update(x) first (the runtime does it
 * inside nb_map_stencil_reduce / nb_cg_*).  Scalar fields. */
nb_status nb_laplace7(const nb_field *x, nb_field *y, nb_view view);
/* <x, y> over all active cells and components, fp64 accumulation in a
 * fixed order that does not depend on the partition count (DESIGN.md
 * "Deterministic reductions").  Synchronises; *host_out receives the value. */
nb_status nb_dot(const nb_field *x, const nb_field *y, double *host_out);
/* The same value written to device memory dev_out (one double, on the grid's
 * device), stream-ordered on the compute stream; does not synchronise. */
nb_status nb_dot_dev(const nb_field *x, const nb_field *y, double *dev_out);

/* Config C1 (Fig. 4a): for k < iters: x <- x + a*y;
 * y <- L(x); dots[k] = <x, y>.  Halo on x (L280).  dots_out: host [iters].
 * Synchronises. */
nb_status nb_map_stencil_reduce(nb_field *x, nb_field *y, double a, int32_t iters, nb_occ occ,
                                double *dots_out);

/* ---- conjugate gradient (Listing 3, UpdateP first L460) ------- */
typedef enum { NB_OP_LAPLACE7 = 0, NB_OP_FEM27 = 1 } nb_operator;
typedef struct {
    int32_t max_iter;     /* iteration cap                                        */
    double rtol;          /* stop when <r,r> <= rtol^2 <r0,r0> (0: fixed count)    */
    nb_occ occ;           /* OCC schedule                                         */
    int32_t check_every;  /* host convergence polling period (iterations)         */
    nb_operator op;       /* A = -L (7-point Poisson) or FEM stiffness K          */
    double fem_E, fem_nu; /* FEM material (op == NB_OP_FEM27)                     */
} nb_cg_params;
typedef struct {
    int32_t iters;        /* iterations performed                                 */
    int32_t converged;    /* 0 running/cap, 1 rtol reached, 2 rr == 0, 3 breakdown */
    double rr0;           /* <r0, r0>                                             */
    double rr;            /* final <r, r>                                         */
} nb_cg_result;
/* Set up r = b - A x, <r,r> on the device (stream-ordered, no sync). */
nb_status nb_cg_create(nb_field *x, const nb_field *b, const nb_cg_params *params, nb_cg **out);
/* Enqueue `iters` CG iterations (graph-launched; converged state turns
 * later iterations into no-ops).  No sync. */
nb_status nb_cg_iterate(nb_cg *cg, int32_t iters);
/* Capture (without running anything) the CUDA graphs that
 * nb_cg_iterate(cg, iters) will launch from the current state, so that the
 * first call does not pay for graph instantiation. */
nb_status nb_cg_prepare(nb_cg *cg, int32_t iters);
/* Apply the deferred x update and read the scalars back.  Synchronises. */
nb_status nb_cg_finish(nb_cg *cg, nb_cg_result *result);
nb_status nb_cg_destroy(nb_cg *cg);
/* create + iterate (polling every check_every) + finish + destroy */
nb_status nb_cg_solve(nb_field *x, const nb_field *b, const nb_cg_params *params,
                      nb_cg_result *result);

/* ---- D3Q19 BGK lattice Boltzmann, twoPop ----------- */
typedef enum { NB_LBM_CAVITY = 0, NB_LBM_PERIODIC = 1 } nb_lbm_bc;
typedef struct {
    double omega;   /* BGK relaxation rate                                     */
    double u_lid;   /* lid velocity (+x) on the face y = Ny (cavity)           */
    double rho_w;   /* wall density in the moving-wall bounce-back term         */
    nb_lbm_bc bc;   /* CAVITY (bounce-back walls + lid) or PERIODIC             */
} nb_lbm_params;
/* f <- equilibrium(rho0, u0); f: fp32 field of cardinality 19 */
nb_status nb_lbm_init(nb_field *f, double rho0, const double u0[3]);
/* nsteps fused pull collide-and-stream steps; *fin and *fout are swapped
 * after every step (twoPop, L451), so on return *fin holds the latest state.
 * Halo: 5 populations per side (c_z = +1 up, c_z = -1 down). */
nb_status nb_lbm_step(nb_field **fin, nb_field **fout, const nb_lbm_params *params,
                      int32_t nsteps, nb_occ occ);
/* AA pattern (PAPER.md L451 stlbm's AA variant): the
 * same physics on ONE population field updated in place (half of twoPop's
 * memory).  Even steps collide locally and store reversed; odd steps pull
 * from and push to the neighbours' opposite slots.  nsteps must be even
 * (NB_EINVAL otherwise) so f returns to the natural layout; the result then
 * equals nsteps twoPop steps bit for bit.  Dense grids, fused halos (one
 * process with virtual partitions, or the peer transport). */
nb_status nb_lbm_step_aa(nb_field *f, const nb_lbm_params *params, int32_t nsteps);
/* rho (card 1) and u (card 3) fp32 fields from f */
nb_status nb_lbm_macroscopic(const nb_field *f, nb_field *rho, nb_field *u);

/* ---- D2Q9 Karman vortex street (Table I; SURVEY.md
 * §8(f) f4).  A dense grid of one plane (Nz = 1), fields fp32 of
 * cardinality 9 (velocities 0; +-x, +-y; (1,1) (-1,-1) (1,-1) (-1,1)).
 * Solid cylinder (x-cx)^2 + (y-cy)^2 <= r^2 (r < 0: none) with half-way
 * bounce-back (solid cells hold 0); bc 0 = channel: y periodic, inflow
 * equilibrium (rho 1, u = (u_in, 0)) for sources left of x = 0,
 * zero-gradient outflow at x = Nx-1; bc 1 = periodic box.  Pull + BGK fused,
 * twoPop (the pointers swap after each step). */
typedef struct {
    double omega, u_in;
    int32_t cx, cy, r, bc;
} nb_d2q9_params;
nb_status nb_d2q9_init(nb_field *f, double rho0, double ux, double uy);
nb_status nb_d2q9_step(nb_field **fin, nb_field **fout, const nb_d2q9_params *params, int32_t nsteps);

/* ---- FEM: Q1 hex linear elasticity, 27-point ------- */
/* y = K u (card 3 fp64), Dirichlet u = 0 on the z = 0 plane (identity
 * rows/cols).  Reads u's halo planes: call nb_halo_update(u) first.
 * Element-sparse grids: nodes = active cells, an
 * element exists iff its 8 nodes are active; y is written at active nodes
 * only.  NB_EMISMATCH unless u, y are fp64 card-3 fields of one grid;
 * NB_EUNSUPPORTED for the AoS layout. */
nb_status nb_fem27_apply(const nb_field *u, nb_field *y, double E, double nu);
/* b = consistent nodal load of pressure p on the top (z = Nz-1) face */
nb_status nb_fem27_rhs(nb_field *b, double pressure);

/* ---- Skeleton (§V) ------------------
 * Sequential user code — a list of Containers — is turned into a data
 * dependency graph (L279-L290: nodes = Containers with operation type,
 * data view and coherency flag; edges = RaW / WaR / WaW on shared data),
 * then a multi-GPU graph (L292-L331: halo-update nodes before incoherent
 * stencils; OCC = NONE / STANDARD (split stencil) / EXTENDED (also the maps
 * before it) / TWO_WAY (also the maps and reduces after it, with the
 * internal -> boundary reduce dependency); transitively redundant edges
 * removed; scheduling hints "launch the internal nodes before the halo"),
 * then a schedule (L333-L396: BFS levels, a stream per concurrent node of
 * the widest level with parent-stream reuse, an event per cross-stream
 * dependency, task order by BFS over data edges + hints).
 * Containers (Listing 3 CG, L154-L163, and the LBM step, L447-L451, are
 * expressible):
 *   AXPBY    y = A x + B y (MapOp).  A = a, or a * s[a_slot] when flags has
 *            NB_SK_A_SLOT (a device scalar: a result slot); B likewise.  Per element:
 *            b == 1 (immediate): fma(A, x, y); a == 1 (immediate) with a
 *            device-scalar B: fma(B, y, x) (UpdateP p = r + beta p);
 *            b == 0 (immediate): A x; otherwise fma(A, x, B y).
 *   LAPLACE7 y = L(x) (StencilOp, 7-point, L = sum of 6 neighbours - 6 x)
 *   POISSON  y = A x = -L(x) = fma(6, x_c, -sum) (StencilOp; the CG operator)
 *   DOT      <x, y> -> slot (ReduceOp, the deterministic dot)
 *   SCALAR   s[slot] = s[x] / s[y] (NB_SC_DIV), s[x] (NB_SC_COPY) or a
 *            (NB_SC_SET): a one-thread device step between reductions
 *            (alpha = rr / pq, beta = rr' / rr, rr = rr'); x, y are slots
 *   LBM      y = D3Q19 BGK pull step of x (StencilOp on fp32 cardinality-19
 *            fields; a = omega, b = u_lid, c = rho_w, sop = bc, CAVITY only);
 *            its halo carries the 5 + 5 z-crossing populations (L256). */
typedef enum {
    NB_SK_AXPBY = 0,
    NB_SK_LAPLACE7 = 1,
    NB_SK_DOT = 2,
    NB_SK_POISSON = 3,
    NB_SK_SCALAR = 4,
    NB_SK_LBM = 5
} nb_container_op;
typedef enum { NB_SC_DIV = 0, NB_SC_COPY = 1, NB_SC_SET = 2 } nb_scalar_op;
typedef struct {
    int32_t op;             /* nb_container_op                                         */
    int32_t x, y;           /* field ids (any non-negative integers naming the data);
                               SCALAR: source slots                                    */
    int32_t slot;           /* DOT / SCALAR: result slot in [0, 1024)                  */
    double a, b;            /* AXPBY coefficients; SCALAR (SET): a; LBM: omega, u_lid   */
    int32_t a_slot, b_slot; /* AXPBY with NB_SK_A_SLOT / NB_SK_B_SLOT: device scalar slots */
    int32_t sop;            /* SCALAR: nb_scalar_op; LBM: nb_lbm_bc                      */
    int32_t flags;          /* NB_SK_A_SLOT | NB_SK_B_SLOT (0: immediate coefficients)   */
    double c;               /* LBM: rho_w                                               */
} nb_container;
#define NB_SK_A_SLOT 1
#define NB_SK_B_SLOT 2
/* Pure host logic (no GPU): plan n containers for an nparts-slab grid and
 * write the plan as JSON into json (cap bytes; json = NULL: only *len) —
 * {"nodes": [{id, name, op, view, container, incoherent, finalize, level,
 * stream, event, waits}], "data": [[from, to]...], "hints": [...],
 * "order": [...], "streams": S, "events": E}. */
nb_status nb_skeleton_plan(int32_t nparts, nb_occ occ, const nb_container *containers, int32_t n, char *json,
                           int64_t cap, int64_t *len);
typedef struct nb_skeleton nb_skeleton;
/* A skeleton over a dense grid; the fields it is given must outlive it, and
 * the grid cannot be destroyed while it lives (NB_ESTATE). */
nb_status nb_skeleton_create(nb_grid *grid, nb_occ occ, nb_skeleton **out);
nb_status nb_skeleton_axpby(nb_skeleton *sk, double a, nb_field *x, double b, nb_field *y);
/* AXPBY with device-scalar coefficients: a_slot / b_slot >= 0 selects a
 * slot (a, b scale it), -1 keeps the immediate (see above) */
nb_status nb_skeleton_axpby_s(nb_skeleton *sk, double a, int32_t a_slot, nb_field *x, double b, int32_t b_slot,
                              nb_field *y);
nb_status nb_skeleton_laplace7(nb_skeleton *sk, nb_field *x, nb_field *y);
nb_status nb_skeleton_poisson(nb_skeleton *sk, nb_field *x, nb_field *y);
nb_status nb_skeleton_dot(nb_skeleton *sk, nb_field *x, nb_field *y, int32_t slot);
nb_status nb_skeleton_scalar(nb_skeleton *sk, nb_scalar_op sop, int32_t in0, int32_t in1, int32_t out, double a);
/* fin, fout: fp32 cardinality-19 fields (twoPop: the next step swaps them) */
nb_status nb_skeleton_lbm(nb_skeleton *sk, nb_field *fin, nb_field *fout, const nb_lbm_params *params);
/* s[slot] = value, stream-ordered on the grid's compute stream */
nb_status nb_skeleton_set_scalar(nb_skeleton *sk, int32_t slot, double value);
/* builds the plan, streams and events (implicit in the first run) */
nb_status nb_skeleton_compile(nb_skeleton *sk);
/* enqueue every task in plan order on its stream (asynchronous; ordered
 * after earlier work on the grid's compute stream, and later work on that
 * stream is ordered after it) */
nb_status nb_skeleton_run(nb_skeleton *sk);
/* a ReduceOp result (synchronises) */
nb_status nb_skeleton_result(nb_skeleton *sk, int32_t slot, double *host);
/* the plan as JSON, as nb_skeleton_plan */
nb_status nb_skeleton_describe(nb_skeleton *sk, char *json, int64_t cap, int64_t *len);
nb_status nb_skeleton_destroy(nb_skeleton *sk);

/* ---- measurement ------------------------------------------------------ */
/* When enabled, every kernel launch is bracketed by CUDA events on the
 * launching stream (graph launch is bypassed).  nb_profile_read
 * synchronises and returns launch count and summed device time of the
 * kernels whose name contains `name`. */
nb_status nb_profile_enable(nb_grid *grid, int32_t enable);
nb_status nb_profile_read(nb_grid *grid, const char *name, int64_t *launches, double *total_ms);
/* Number of this library's kernels launched on the grid since creation
 * (graph launches count their kernel nodes). */
nb_status nb_launch_count(const nb_grid *grid, int64_t *count);

#ifdef __cplusplus
}
#endif
#endif /* NB_H */
