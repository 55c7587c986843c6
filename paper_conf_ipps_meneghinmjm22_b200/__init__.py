"""B200-native Neon map-stencil hot path — thin Python binding over libnb.so.

Argument marshalling only: every step of the path runs in the CUDA kernels
of ``libnb.so`` (sm_100a), declared in ``include/nb.h``.  The functions keep
the C names (``nb_axpy``, ``nb_laplace7``, ``nb_cg_solve`` ...); ``Grid`` and
``Field`` own the opaque handles.  There is no CPU fallback: importing works
on any host, but every call that needs a GPU raises ``NbError`` (status
NB_ECUDA) without one, and a missing ``libnb.so`` raises ``ImportError`` on
first use.

Paper: Meneghin et al., "Neon: A Multi-GPU Programming Model for Grid-based
Computations", IPDPS 2022.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

__all__ = [
    "NbError", "Grid", "Field", "CG", "Comm", "lib", "LIB_PATH",
    "NB_F32", "NB_F64", "VIEW_STANDARD", "VIEW_INTERNAL", "VIEW_BOUNDARY",
    "OCC_NONE", "OCC_STANDARD", "OCC_EXTENDED", "OCC_TWO_WAY",
]

LIB_PATH = os.environ.get("NB_LIB") or os.path.join(os.path.dirname(os.path.abspath(__file__)), "libnb.so")

NB_OK, NB_EINVAL, NB_ENOMEM, NB_ECUDA, NB_ENCCL, NB_EMISMATCH, NB_EUNSUPPORTED, NB_ESTATE = range(8)
NB_F32, NB_F64 = 0, 1
VIEW_STANDARD, VIEW_INTERNAL, VIEW_BOUNDARY = 0, 1, 2
OCC_NONE, OCC_STANDARD, OCC_EXTENDED, OCC_TWO_WAY = 0, 1, 2, 3
FILL_CONST, FILL_UNIFORM, FILL_INT_UNIFORM, FILL_POISSON_RHS = 0, 1, 2, 3
OP_LAPLACE7, OP_FEM27 = 0, 1
LBM_CAVITY, LBM_PERIODIC = 0, 1
HALO_FUSED, HALO_STREAM = 0, 1
SOA, SOA_PLANE, AOS = 0, 1, 2  # field layouts (include/nb.h nb_layout)
OCC_NAMES = {"none": OCC_NONE, "standard": OCC_STANDARD, "extended": OCC_EXTENDED, "two_way": OCC_TWO_WAY}


class NbError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"[nb status {status}] {msg}")
        self.status = status


class PartInfo(C.Structure):
    _fields_ = [("device", C.c_int32), ("local", C.c_int32), ("z_begin", C.c_int32), ("z_end", C.c_int32),
                ("n_cells", C.c_int64), ("n_bnd_lo", C.c_int64), ("n_bnd_hi", C.c_int64),
                ("n_internal", C.c_int64)]


class CgParams(C.Structure):
    _fields_ = [("max_iter", C.c_int32), ("rtol", C.c_double), ("occ", C.c_int32),
                ("check_every", C.c_int32), ("op", C.c_int32), ("fem_E", C.c_double), ("fem_nu", C.c_double)]


class CgResult(C.Structure):
    _fields_ = [("iters", C.c_int32), ("converged", C.c_int32), ("rr0", C.c_double), ("rr", C.c_double)]


class LbmParams(C.Structure):
    _fields_ = [("omega", C.c_double), ("u_lid", C.c_double), ("rho_w", C.c_double), ("bc", C.c_int32)]


class Container(C.Structure):
    _fields_ = [("op", C.c_int32), ("x", C.c_int32), ("y", C.c_int32), ("slot", C.c_int32),
                ("a", C.c_double), ("b", C.c_double), ("a_slot", C.c_int32), ("b_slot", C.c_int32),
                ("sop", C.c_int32), ("flags", C.c_int32), ("c", C.c_double)]


SK_AXPBY, SK_LAPLACE7, SK_DOT, SK_POISSON, SK_SCALAR, SK_LBM = 0, 1, 2, 3, 4, 5
SC_DIV, SC_COPY, SC_SET = 0, 1, 2
SK_A_SLOT, SK_B_SLOT = 1, 2


# exported symbols and their ctypes signatures (the whole of include/nb.h)
P, I32, I64, D, U64 = C.c_void_p, C.c_int32, C.c_int64, C.c_double, C.c_uint64
PP = C.POINTER(C.c_void_p)
SIGNATURES = {
    "nb_version": ([], C.c_char_p),
    "nb_last_error": ([], C.c_char_p),
    "nb_device_count": ([], I32),
    "nb_comm_unique_id": ([P], I32),
    "nb_comm_create": ([I32, I32, P, I32, PP], I32),
    "nb_comm_destroy": ([P], I32),
    "nb_comm_create_peer": ([I32, I32, I32, P, P, PP], I32),
    "nb_comm_is_peer": ([P, P], I32),
    "nb_partition_plan": ([I32, I32, P], I32),
    "nb_partition_plan_weighted": ([I32, P, I32, P], I32),
    "nb_halo_plan": ([I32, I32, I32, I32, I32, P, I32, P], I32),
    "nb_grid_create_dense": ([P, I32, P, P, PP], I32),
    "nb_grid_create_sparse": ([P, P, I32, P, P, PP], I32),
    "nb_grid_destroy": ([P], I32),
    "nb_grid_num_partitions": ([P, P], I32),
    "nb_grid_partition_info": ([P, I32, P], I32),
    "nb_grid_set_streams": ([P, P, P], I32),
    "nb_grid_get_stream": ([P, PP], I32),
    "nb_sync": ([P], I32),
    "nb_grid_trim": ([P, P], I32),
    "nb_grid_set_halo_mode": ([P, I32], I32),
    "nb_field_create": ([P, I32, I32, I32, D, PP], I32),
    "nb_field_layout": ([P, P], I32),
    "nb_field_destroy": ([P], I32),
    "nb_field_required_elems": ([P, I32, I32, P], I32),
    "nb_field_wrap": ([P, I32, I32, I32, D, P, PP], I32),
    "nb_field_upload": ([P, P, I64], I32),
    "nb_field_download": ([P, P, I64], I32),
    "nb_field_fill": ([P, I32, U64, D, D], I32),
    "nb_halo_update": ([P], I32),
    "nb_field_partition_ptr": ([P, I32, PP, P, P, P], I32),
    "nb_axpy": ([D, P, P, I32], I32),
    "nb_axpby": ([D, P, D, P, I32], I32),
    "nb_laplace7": ([P, P, I32], I32),
    "nb_dot": ([P, P, P], I32),
    "nb_dot_dev": ([P, P, P], I32),
    "nb_map_stencil_reduce": ([P, P, D, I32, I32, P], I32),
    "nb_cg_create": ([P, P, P, PP], I32),
    "nb_cg_iterate": ([P, I32], I32),
    "nb_cg_prepare": ([P, I32], I32),
    "nb_cg_finish": ([P, P], I32),
    "nb_cg_destroy": ([P], I32),
    "nb_cg_solve": ([P, P, P, P], I32),
    "nb_lbm_init": ([P, D, P], I32),
    "nb_lbm_step": ([PP, PP, P, I32, I32], I32),
    "nb_lbm_macroscopic": ([P, P, P], I32),
    "nb_lbm_step_aa": ([P, P, I32], I32),
    "nb_d2q9_init": ([P, D, D, D], I32),
    "nb_d2q9_step": ([PP, PP, P, I32], I32),
    "nb_fem27_apply": ([P, P, D, D], I32),
    "nb_fem27_rhs": ([P, D], I32),
    "nb_skeleton_plan": ([I32, I32, P, I32, P, I64, P], I32),
    "nb_skeleton_create": ([P, I32, PP], I32),
    "nb_skeleton_axpby": ([P, D, P, D, P], I32),
    "nb_skeleton_axpby_s": ([P, D, I32, P, D, I32, P], I32),
    "nb_skeleton_laplace7": ([P, P, P], I32),
    "nb_skeleton_poisson": ([P, P, P], I32),
    "nb_skeleton_dot": ([P, P, P, I32], I32),
    "nb_skeleton_scalar": ([P, I32, I32, I32, I32, D], I32),
    "nb_skeleton_lbm": ([P, P, P, P], I32),
    "nb_skeleton_set_scalar": ([P, I32, D], I32),
    "nb_skeleton_compile": ([P], I32),
    "nb_skeleton_run": ([P], I32),
    "nb_skeleton_result": ([P, I32, P], I32),
    "nb_skeleton_describe": ([P, P, I64, P], I32),
    "nb_skeleton_destroy": ([P], I32),
    "nb_profile_enable": ([P, I32], I32),
    "nb_profile_read": ([P, C.c_char_p, P, P], I32),
    "nb_launch_count": ([P, P], I32),
}

_lib = None


def lib():
    """Load libnb.so (loudly: ImportError if it was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() "
                              "(python -m paper_conf_ipps_meneghinmjm22_b200.build)")
        L = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)
        for name, (args, res) in SIGNATURES.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _lib = L
    return _lib


def _check(status: int) -> None:
    if status != NB_OK:
        raise NbError(status, lib().nb_last_error().decode(errors="replace"))


def _h(obj):
    return obj.handle if hasattr(obj, "handle") else obj


_DT = {NB_F32: np.float32, NB_F64: np.float64, "f32": NB_F32, "f64": NB_F64,
       np.float32: NB_F32, np.float64: NB_F64}


def _dtype_code(dt) -> int:
    if isinstance(dt, int):
        return dt
    if isinstance(dt, str):
        return _DT[dt]
    return _DT[np.dtype(dt).type]


def nb_version() -> str:
    return lib().nb_version().decode()


def nb_device_count() -> int:
    return int(lib().nb_device_count())


def nb_partition_plan(nz: int, nparts: int) -> list:
    zb = (C.c_int32 * (nparts + 1))()
    _check(lib().nb_partition_plan(nz, nparts, zb))
    return list(zb)


def nb_partition_plan_weighted(counts, nparts: int) -> list:
    c = np.ascontiguousarray(counts, dtype=np.int64)
    zb = (C.c_int32 * (nparts + 1))()
    _check(lib().nb_partition_plan_weighted(len(c), c.ctypes.data_as(P), nparts, zb))
    return list(zb)


class HaloMsg(C.Structure):
    _fields_ = [("src_part", C.c_int32), ("dst_part", C.c_int32), ("src_rank", C.c_int32),
                ("dst_rank", C.c_int32), ("src_plane", C.c_int32), ("dst_plane", C.c_int32), ("up", C.c_int32)]


def nb_halo_plan(nz: int, nparts: int, world: int = 1, rank: int = -1, periodic: bool = False) -> list:
    """Halo messages (dicts) this rank posts, in the canonical order."""
    n = C.c_int32()
    _check(lib().nb_halo_plan(nz, nparts, world, rank, int(periodic), None, 0, C.byref(n)))
    arr = (HaloMsg * max(n.value, 1))()
    _check(lib().nb_halo_plan(nz, nparts, world, rank, int(periodic), arr, n.value, C.byref(n)))
    return [{k: getattr(m, k) for k, _ in HaloMsg._fields_} for m in arr[:n.value]]


# ---------------------------------------------------------------------------
# host allgather callback of the peer-memory transport (include/nb.h)
ALLGATHER_FN = C.CFUNCTYPE(C.c_int32, C.c_void_p, C.c_void_p, C.c_int64, C.c_void_p)


def _torch_allgather(world: int, group):
    """nb_allgather_fn over a CPU (gloo) torch.distributed group: setup-time
    plumbing only (IPC handles, teardown barriers), never on the data path."""
    import traceback

    import torch
    import torch.distributed as dist

    def ag(ctx, send, nbytes, recv):
        try:
            mine = torch.frombuffer(bytearray(C.string_at(send, nbytes)), dtype=torch.uint8)
            outs = [torch.empty(nbytes, dtype=torch.uint8) for _ in range(world)]
            dist.all_gather(outs, mine, group=group)
            data = b"".join(o.numpy().tobytes() for o in outs)
            C.memmove(recv, data, len(data))
            return 0
        except Exception:  # reported to libnb as a failed collective
            traceback.print_exc()
            return 1

    return ALLGATHER_FN(ag)


class Comm:
    """One process per GPU.  transport="peer" (default): libnb's
    peer-memory transport — CUDA IPC mappings of the neighbours' halos and of
    every rank's reduction buffer, kernels store across GPUs and signal with
    device flags; torch.distributed (gloo) only exchanges IPC handles at
    setup.  transport="nccl": an NCCL communicator inside libnb (the 128-byte
    unique id is broadcast with torch.distributed)."""

    def __init__(self, world: int, rank: int, device: int, uid: bytes | None = None, allgather=None):
        self.handle = P()
        self._ag = None
        if allgather is not None:
            self._ag = allgather  # keep the callback alive as long as the comm
            _check(lib().nb_comm_create_peer(world, rank, device, C.cast(allgather, C.c_void_p), None,
                                             C.byref(self.handle)))
            self.transport = "peer"
        else:
            buf = (C.c_uint8 * 128).from_buffer_copy(uid)
            _check(lib().nb_comm_create(world, rank, buf, device, C.byref(self.handle)))
            self.transport = "nccl"
        self.world, self.rank, self.device = world, rank, device

    @staticmethod
    def unique_id() -> bytes:
        buf = (C.c_uint8 * 128)()
        _check(lib().nb_comm_unique_id(buf))
        return bytes(buf)

    @classmethod
    def from_torch_distributed(cls, device: int, transport: str | None = None):
        """Build the communicator of the current torch.distributed world;
        transport defaults to $NB_TRANSPORT or "peer"."""
        import torch.distributed as dist
        transport = transport or os.environ.get("NB_TRANSPORT", "peer")
        world, rank = dist.get_world_size(), dist.get_rank()
        if transport == "peer":
            group = dist.new_group(backend="gloo") if dist.get_backend() != "gloo" else None
            comm = cls(world, rank, device, allgather=_torch_allgather(world, group))
            comm._group = group
            return comm
        if transport != "nccl":
            raise ValueError(f"transport must be 'peer' or 'nccl', got {transport!r}")
        uid = [cls.unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        return cls(world, rank, device, uid[0])

    def close(self):
        if self.handle:
            _check(lib().nb_comm_destroy(self.handle))
            self.handle = P()


class Grid:
    """Dense or element-sparse grid split into z-slabs."""

    def __init__(self, dims, nparts: int = 1, devices=None, comm: Comm | None = None, active=None):
        self.dims = tuple(int(d) for d in dims)
        self.nparts = int(nparts)
        d = (C.c_int32 * 3)(*self.dims)
        if comm is None:
            devs = [0] * self.nparts if devices is None else list(devices)
            dv = (C.c_int32 * self.nparts)(*devs)
            self.device = int(devs[0])
        else:
            self.device = int(comm.device)
            k = self.nparts // comm.world
            dv = (C.c_int32 * max(k, 1))(*([comm.device] * max(k, 1)))
        self.handle = P()
        self.comm = comm
        self.sparse = active is not None
        if active is None:
            _check(lib().nb_grid_create_dense(d, self.nparts, dv, _h(comm) if comm else None,
                                              C.byref(self.handle)))
        else:
            a = np.ascontiguousarray(active, dtype=np.uint8)
            assert a.shape == self.dims[::-1], "active mask is [z][y][x]"
            self._active = a
            _check(lib().nb_grid_create_sparse(d, a.ctypes.data_as(P), self.nparts, dv,
                                               _h(comm) if comm else None, C.byref(self.handle)))

    @property
    def ncells(self) -> int:
        return self.dims[0] * self.dims[1] * self.dims[2]

    def partition_info(self, g: int) -> dict:
        pi = PartInfo()
        _check(lib().nb_grid_partition_info(self.handle, g, C.byref(pi)))
        return {k: getattr(pi, k) for k, _ in PartInfo._fields_}

    def set_streams(self, compute=None, halo=None):
        _check(lib().nb_grid_set_streams(self.handle, compute, halo))

    def stream(self) -> int:
        s = P()
        _check(lib().nb_grid_get_stream(self.handle, C.byref(s)))
        return s.value or 0

    def sync(self):
        _check(lib().nb_sync(self.handle))

    def trim(self) -> int:
        """Free the cached device buffers of destroyed fields; returns bytes."""
        n = C.c_int64()
        _check(lib().nb_grid_trim(self.handle, C.byref(n)))
        return n.value

    def set_halo_mode(self, mode: int):
        """HALO_FUSED (stores from the boundary kernels) or HALO_STREAM
        (device copies on the halo stream, overlapped with the interior)."""
        _check(lib().nb_grid_set_halo_mode(self.handle, int(mode)))

    def launch_count(self) -> int:
        n = C.c_int64()
        _check(lib().nb_launch_count(self.handle, C.byref(n)))
        return n.value

    def profile(self, enable: bool = True):
        _check(lib().nb_profile_enable(self.handle, int(enable)))

    def profile_read(self, name: str):
        n, ms = C.c_int64(), C.c_double()
        _check(lib().nb_profile_read(self.handle, name.encode(), C.byref(n), C.byref(ms)))
        return n.value, ms.value

    def close(self):
        if self.handle:
            _check(lib().nb_grid_destroy(self.handle))
            self.handle = P()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


class Field:
    """Field of `card` components (PAPER.md L58-L63 newField<T>(cardinality,
    outsideDomainValue)) with z halo planes, in layout SOA (default),
    SOA_PLANE or AOS (L248; include/nb.h)."""

    def __init__(self, grid: Grid, dtype="f64", card: int = 1, outside: float = 0.0, _buffers=None,
                 layout: int = 0):
        self.grid = grid
        self.dt = _dtype_code(dtype)
        self.np_dtype = _DT[self.dt]
        self.card = int(card)
        self.outside = float(outside)
        self.handle = P()
        self.buffers = _buffers  # borrowed storage (kept alive with the field)
        if _buffers is None:
            _check(lib().nb_field_create(grid.handle, self.dt, self.card, int(layout), self.outside,
                                         C.byref(self.handle)))
        else:
            ptrs = (C.c_void_p * len(_buffers))(*[b.data_ptr() for b in _buffers])
            _check(lib().nb_field_wrap(grid.handle, self.dt, self.card, int(layout), self.outside, ptrs,
                                       C.byref(self.handle)))

    @property
    def layout(self) -> int:
        v = C.c_int32()
        _check(lib().nb_field_layout(self.handle, C.byref(v)))
        return v.value

    @staticmethod
    def required_elems(grid: Grid, card: int, part: int) -> int:
        n = C.c_int64()
        _check(lib().nb_field_required_elems(grid.handle, int(card), int(part), C.byref(n)))
        return n.value

    @classmethod
    def wrap(cls, grid: Grid, buffers, dtype="f64", card: int = 1, outside: float = 0.0, layout: int = 0):
        """Field over caller-owned torch CUDA tensors, one per local partition
        (each >= required_elems elements; torch keeps ownership)."""
        return cls(grid, dtype, card, outside, _buffers=list(buffers), layout=layout)

    @classmethod
    def empty_torch(cls, grid: Grid, dtype="f64", card: int = 1, outside: float = 0.0, layout: int = 0):
        """Allocate the partitions with torch.empty on the grid's device and wrap them."""
        import torch
        tdt = torch.float64 if _dtype_code(dtype) == 1 else torch.float32
        dev = torch.device("cuda", grid.device)
        bufs = [torch.empty(cls.required_elems(grid, card, p), dtype=tdt, device=dev)
                for p in range(grid.nparts) if grid.partition_info(p)["local"]]
        return cls.wrap(grid, bufs, dtype, card, outside, layout)

    @property
    def shape(self):
        nx, ny, nz = self.grid.dims
        return (nz, ny, nx) if self.card == 1 else (self.card, nz, ny, nx)

    @property
    def nbytes(self) -> int:
        return int(np.prod(self.shape)) * np.dtype(self.np_dtype).itemsize

    def upload(self, host) -> None:
        """host: numpy array (dense logical view) or a pinned CPU torch tensor."""
        if hasattr(host, "data_ptr"):  # torch tensor (pinned for the e2e path)
            assert host.numel() * host.element_size() == self.nbytes
            _check(lib().nb_field_upload(self.handle, P(host.data_ptr()), self.nbytes))
            self.grid.sync()
            return
        a = np.ascontiguousarray(host, dtype=self.np_dtype)
        assert a.size * a.itemsize == self.nbytes, (a.shape, self.shape)
        _check(lib().nb_field_upload(self.handle, a.ctypes.data_as(P), a.nbytes))
        self.grid.sync()  # the host buffer is borrowed until the copy completes

    def upload_async(self, ptr: int) -> None:
        _check(lib().nb_field_upload(self.handle, P(ptr), self.nbytes))

    def download(self, out=None):
        if out is not None and hasattr(out, "data_ptr"):
            _check(lib().nb_field_download(self.handle, P(out.data_ptr()), self.nbytes))
            return out
        a = np.empty(self.shape, dtype=self.np_dtype) if out is None else out
        _check(lib().nb_field_download(self.handle, a.ctypes.data_as(P), self.nbytes))
        return a

    def fill(self, kind: int, seed: int = 0, a: float = 0.0, b: float = 0.0):
        _check(lib().nb_field_fill(self.handle, kind, seed, a, b))

    def fill_uniform(self, seed=1, lo=-1.0, hi=1.0):
        self.fill(FILL_UNIFORM, seed, lo, hi)

    def fill_int(self, seed=1, lo=-8, hi=8):
        self.fill(FILL_INT_UNIFORM, seed, lo, hi)

    def fill_const(self, v):
        self.fill(FILL_CONST, 0, v, 0.0)

    def halo_update(self):
        _check(lib().nb_halo_update(self.handle))

    def partition_ptr(self, g: int):
        p, pitch, ps, cs = P(), C.c_int64(), C.c_int64(), C.c_int64()
        _check(lib().nb_field_partition_ptr(self.handle, g, C.byref(p), C.byref(pitch), C.byref(ps),
                                            C.byref(cs)))
        return p.value, pitch.value, ps.value, cs.value

    def close(self):
        if self.handle:
            _check(lib().nb_field_destroy(self.handle))
            self.handle = P()


# ---- ops (same names as the C ABI) -----------------------------------------
def nb_axpy(a: float, x: Field, y: Field, view: int = VIEW_STANDARD):
    _check(lib().nb_axpy(a, _h(x), _h(y), view))


def nb_axpby(a: float, x: Field, b: float, y: Field, view: int = VIEW_STANDARD):
    _check(lib().nb_axpby(a, _h(x), b, _h(y), view))


def nb_laplace7(x: Field, y: Field, view: int = VIEW_STANDARD):
    _check(lib().nb_laplace7(_h(x), _h(y), view))


def nb_halo_update(f: Field):
    _check(lib().nb_halo_update(_h(f)))


def nb_dot(x: Field, y: Field) -> float:
    out = C.c_double()
    _check(lib().nb_dot(_h(x), _h(y), C.byref(out)))
    return out.value


def nb_dot_dev(x: Field, y: Field, out_ptr: int) -> None:
    """<x, y> written to the device double at out_ptr (e.g. a torch tensor's
    data_ptr()), stream-ordered; no synchronisation."""
    _check(lib().nb_dot_dev(_h(x), _h(y), P(out_ptr)))


def nb_map_stencil_reduce(x: Field, y: Field, a: float = 0.125, iters: int = 10, occ: int = OCC_TWO_WAY):
    dots = np.zeros(max(iters, 1), dtype=np.float64)
    _check(lib().nb_map_stencil_reduce(_h(x), _h(y), a, iters, occ, dots.ctypes.data_as(P)))
    return dots[:iters]


def _cg_params(max_iter, rtol, occ, check_every, op, E, nu):
    return CgParams(int(max_iter), float(rtol), int(occ), int(check_every), int(op), float(E), float(nu))


class CG:
    """Matrix-free CG (Listing 3, UpdateP first L460) driven on the device."""

    def __init__(self, x: Field, b: Field, max_iter=100, rtol=0.0, occ=OCC_TWO_WAY, check_every=16,
                 op=OP_LAPLACE7, E=1.0, nu=0.3):
        self.prm = _cg_params(max_iter, rtol, occ, check_every, op, E, nu)
        self.handle = P()
        _check(lib().nb_cg_create(_h(x), _h(b), C.byref(self.prm), C.byref(self.handle)))

    def iterate(self, n: int):
        _check(lib().nb_cg_iterate(self.handle, int(n)))

    def prepare(self, n: int):
        """Build the CUDA graphs iterate(n) will launch (no GPU work)."""
        _check(lib().nb_cg_prepare(self.handle, int(n)))

    def finish(self) -> CgResult:
        r = CgResult()
        _check(lib().nb_cg_finish(self.handle, C.byref(r)))
        return r

    def close(self):
        if self.handle:
            _check(lib().nb_cg_destroy(self.handle))
            self.handle = P()


def nb_cg_solve(x: Field, b: Field, max_iter=100, rtol=0.0, occ=OCC_TWO_WAY, check_every=16,
                op=OP_LAPLACE7, E=1.0, nu=0.3) -> CgResult:
    prm = _cg_params(max_iter, rtol, occ, check_every, op, E, nu)
    r = CgResult()
    _check(lib().nb_cg_solve(_h(x), _h(b), C.byref(prm), C.byref(r)))
    return r


def nb_lbm_init(f: Field, rho0: float = 1.0, u0=(0.0, 0.0, 0.0)):
    u = (C.c_double * 3)(*u0)
    _check(lib().nb_lbm_init(_h(f), rho0, u))


def nb_lbm_step(fin: Field, fout: Field, omega: float, nsteps: int = 1, u_lid: float = 0.05,
                rho_w: float = 1.0, bc: int = LBM_CAVITY, occ: int = OCC_STANDARD):
    """Returns (fin, fout) after the swaps: fin holds the latest state."""
    prm = LbmParams(omega, u_lid, rho_w, bc)
    a, b = P(fin.handle.value), P(fout.handle.value)
    _check(lib().nb_lbm_step(C.byref(a), C.byref(b), C.byref(prm), int(nsteps), int(occ)))
    if a.value == fin.handle.value:
        return fin, fout
    return fout, fin


def nb_lbm_step_aa(f: Field, omega: float, nsteps: int = 2, u_lid: float = 0.05, rho_w: float = 1.0,
                   bc: int = LBM_CAVITY):
    """AA pattern: nsteps (even) steps in place on ONE population field."""
    prm = LbmParams(omega, u_lid, rho_w, bc)
    _check(lib().nb_lbm_step_aa(_h(f), C.byref(prm), int(nsteps)))
    return f


class D2q9Params(C.Structure):
    _fields_ = [("omega", C.c_double), ("u_in", C.c_double), ("cx", C.c_int32), ("cy", C.c_int32),
                ("r", C.c_int32), ("bc", C.c_int32)]


D2Q9_CHANNEL, D2Q9_PERIODIC = 0, 1


def nb_d2q9_init(f: Field, rho0: float = 1.0, ux: float = 0.0, uy: float = 0.0):
    _check(lib().nb_d2q9_init(_h(f), rho0, ux, uy))


def nb_d2q9_step(fin: Field, fout: Field, omega: float, u_in: float, cyl=(0, 0, -1), nsteps: int = 1,
                 bc: int = D2Q9_CHANNEL):
    """Kármán vortex street step(s); returns (fin, fout) after the swaps."""
    prm = D2q9Params(omega, u_in, int(cyl[0]), int(cyl[1]), int(cyl[2]), int(bc))
    a, b = P(fin.handle.value), P(fout.handle.value)
    _check(lib().nb_d2q9_step(C.byref(a), C.byref(b), C.byref(prm), int(nsteps)))
    return (fin, fout) if a.value == fin.handle.value else (fout, fin)


def nb_lbm_macroscopic(f: Field, rho: Field, u: Field):
    _check(lib().nb_lbm_macroscopic(_h(f), _h(rho), _h(u)))


def nb_fem27_apply(u: Field, y: Field, E: float = 1.0, nu: float = 0.3):
    _check(lib().nb_fem27_apply(_h(u), _h(y), E, nu))


def nb_fem27_rhs(b: Field, pressure: float = 1.0):
    _check(lib().nb_fem27_rhs(_h(b), pressure))


# ---- Skeleton (§V): sequential containers -> graph -> schedule ----
def _json_out(call):
    import json
    n = C.c_int64()
    _check(call(None, 0, C.byref(n)))
    buf = C.create_string_buffer(n.value + 1)
    _check(call(buf, n.value + 1, C.byref(n)))
    return json.loads(buf.value.decode())


def nb_skeleton_plan(nparts: int, occ: int, containers) -> dict:
    """Pure host planning (no GPU).  containers: (op, x, y, a, b, slot)
    tuples with integer field ids, optionally followed by (a_slot, b_slot,
    sop): device-scalar coefficient slots (-1: immediate) and the scalar op;
    returns the plan (nodes, data edges, hints, task order, streams,
    events)."""
    arr = (Container * max(len(containers), 1))()
    for i, t in enumerate(containers):
        op, x, y, a, b, slot = t[:6]
        a_slot, b_slot, sop = (tuple(t[6:9]) + (-1, -1, 0)[len(t[6:9]):])
        flags = (SK_A_SLOT if a_slot >= 0 else 0) | (SK_B_SLOT if b_slot >= 0 else 0)
        arr[i] = Container(op, x, y, slot, a, b, a_slot, b_slot, sop, flags, 0.0)
    return _json_out(lambda buf, cap, n: lib().nb_skeleton_plan(int(nparts), int(occ), arr, len(containers),
                                                                 buf, cap, n))


class Skeleton:
    """Sequential user code over fields, executed by the Skeleton's
    generated multi-GPU schedule (§V)."""

    def __init__(self, grid: Grid, occ: int = OCC_TWO_WAY):
        self.grid = grid
        self.handle = P()
        self.fields = []  # keep the fields alive as long as the skeleton
        _check(lib().nb_skeleton_create(grid.handle, int(occ), C.byref(self.handle)))

    def axpby(self, a: float, x: Field, b: float, y: Field):
        self.fields += [x, y]
        _check(lib().nb_skeleton_axpby(self.handle, float(a), _h(x), float(b), _h(y)))

    def axpy(self, a: float, x: Field, y: Field):
        self.axpby(a, x, 1.0, y)

    def axpby_s(self, a: float, a_slot: int, x: Field, b: float, b_slot: int, y: Field):
        """y = A x + B y with A = a * s[a_slot] (a_slot >= 0) or a, B likewise."""
        self.fields += [x, y]
        _check(lib().nb_skeleton_axpby_s(self.handle, float(a), int(a_slot), _h(x), float(b), int(b_slot), _h(y)))

    def laplace7(self, x: Field, y: Field):
        self.fields += [x, y]
        _check(lib().nb_skeleton_laplace7(self.handle, _h(x), _h(y)))

    def poisson(self, x: Field, y: Field):
        """y = A x = -L(x) (the CG operator)."""
        self.fields += [x, y]
        _check(lib().nb_skeleton_poisson(self.handle, _h(x), _h(y)))

    def scalar(self, sop: int, in0: int, in1: int, out: int, a: float = 0.0):
        _check(lib().nb_skeleton_scalar(self.handle, int(sop), int(in0), int(in1), int(out), float(a)))

    def lbm(self, fin: Field, fout: Field, omega: float, u_lid: float = 0.05, rho_w: float = 1.0):
        self.fields += [fin, fout]
        prm = LbmParams(omega, u_lid, rho_w, LBM_CAVITY)
        _check(lib().nb_skeleton_lbm(self.handle, _h(fin), _h(fout), C.byref(prm)))

    def set_scalar(self, slot: int, value: float):
        _check(lib().nb_skeleton_set_scalar(self.handle, int(slot), float(value)))

    def dot(self, x: Field, y: Field, slot: int):
        self.fields += [x, y]
        _check(lib().nb_skeleton_dot(self.handle, _h(x), _h(y), int(slot)))

    def compile(self):
        _check(lib().nb_skeleton_compile(self.handle))

    def run(self):
        _check(lib().nb_skeleton_run(self.handle))

    def result(self, slot: int) -> float:
        v = C.c_double()
        _check(lib().nb_skeleton_result(self.handle, int(slot), C.byref(v)))
        return v.value

    def describe(self) -> dict:
        return _json_out(lambda buf, cap, n: lib().nb_skeleton_describe(self.handle, buf, cap, n))

    def close(self):
        if self.handle:
            _check(lib().nb_skeleton_destroy(self.handle))
            self.handle = P()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
