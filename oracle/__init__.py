"""CPU oracle for the Neon map-stencil hot path — TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and the ``cpu_baseline`` /
``--impl reference`` legs of ``bench.py`` may import this package.  The
product path (``paper_conf_ipps_meneghinmjm22_b200``) never imports it, and
this package never imports the product path: the two share no code.

The arithmetic lives in ``oracle.c`` (plain C, fp64, -ffp-contract=off),
compiled on first use into ``oracle/liboracle.so``; this module only
marshals numpy arrays.  Every function cites its PAPER.md passage in
``oracle.c``.  Pins: ``tests/test_oracle_*.py``.  Functions without a pin
are marked "parity unpinned" here and in DESIGN.md (none at present).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
CFLAGS = ["-O2", "-std=c11", "-fPIC", "-shared", "-fopenmp", "-ffp-contract=off",
          "-fno-fast-math", "-Wall"]


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        P = C.c_void_p
        i64, i32, d = C.c_int64, C.c_int, C.c_double
        L.or_axpy.argtypes = [i64, d, P, P]
        L.or_axpby.argtypes = [i64, d, P, d, P]
        L.or_dot.argtypes = [i64, P, P]
        L.or_dot.restype = d
        L.or_dot_planes.argtypes = [i64, i64, P, P]
        L.or_dot_planes.restype = d
        L.or_laplace7.argtypes = [i32, i32, i32, d, P, P]
        L.or_sparse_laplace7.argtypes = [i32, i32, i32, P, d, P, P]
        L.or_c1_loop.argtypes = [i32, i32, i32, d, i32, P, P, P]
        L.or_fem_ke.argtypes = [d, d, P]
        L.or_fem_apply.argtypes = [i32, i32, i32, P, P, i32, P, P]
        L.or_fem_rhs.argtypes = [i32, i32, i32, P, i32, d, P]
        L.or_cg.argtypes = [i32, i32, i32, i32, P, P, P, P, i32, d, P, P]
        L.or_cg.restype = i32
        L.or_lbm_lattice.argtypes = [P, P, P]
        L.or_lbm_step.argtypes = [i32, i32, i32, i32, d, d, d, P, P]
        L.or_lbm_step_masked.argtypes = [i32, i32, i32, i32, d, d, d, P, P, P]
        L.or_d2q9_lattice.argtypes = [P, P, P]
        L.or_d2q9_step.argtypes = [i32, i32, i32, d, d, i32, i32, i32, P, P]
        L.or_lbm_macroscopic.argtypes = [i32, i32, i32, P, P, P]
        L.or_num_threads.restype = i32
        L.or_set_num_threads.argtypes = [i32]
        _lib = L
    return _lib


class CGResult(C.Structure):
    _fields_ = [("iters", C.c_int32), ("converged", C.c_int32), ("rr0", C.c_double),
                ("rr", C.c_double)]


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def _ptr(a):
    return a.ctypes.data_as(C.c_void_p)


def num_threads() -> int:
    return lib().or_num_threads()


def set_num_threads(n: int) -> None:
    lib().or_set_num_threads(int(n))


# ---- maps (PAPER.md eq. L104) -------------------------------------------
def axpy(a, x, y):
    """returns a*x + y"""
    x = _f64(x)
    y = _f64(y).copy()
    lib().or_axpy(x.size, float(a), _ptr(x), _ptr(y))
    return y


def axpby(a, x, b, y):
    x = _f64(x)
    y = _f64(y).copy()
    lib().or_axpby(x.size, float(a), _ptr(x), float(b), _ptr(y))
    return y


# ---- reduce (PAPER.md eq. L129) -----------------------------------------
def dot(x, y) -> float:
    """Nearly correctly rounded sum_i x_i y_i (double-double accumulation)."""
    x = _f64(x)
    y = _f64(y)
    return lib().or_dot(x.size, _ptr(x), _ptr(y))


# ---- stencils ---------------------------------
def laplace7(x, outside: float = 0.0):
    """x: [z][y][x] fp64 -> L(x) with out-of-domain neighbours = outside."""
    x = _f64(x)
    nz, ny, nx = x.shape
    y = np.empty_like(x)
    lib().or_laplace7(nx, ny, nz, float(outside), _ptr(x), _ptr(y))
    return y


def sparse_laplace7(mask, x, outside: float = 0.0):
    x = _f64(x)
    m = np.ascontiguousarray(mask, dtype=np.uint8)
    nz, ny, nx = x.shape
    y = np.empty_like(x)
    lib().or_sparse_laplace7(nx, ny, nz, _ptr(m), float(outside), _ptr(x), _ptr(y))
    return y


def c1_loop(x0, a: float = 0.125, iters: int = 10, y0=None):
    """Config C1 (Fig. 4a): returns (x, y, dots[iters])."""
    x = _f64(x0).copy()
    y = np.zeros_like(x) if y0 is None else _f64(y0).copy()
    nz, ny, nx = x.shape
    dots = np.zeros(iters, dtype=np.float64)
    lib().or_c1_loop(nx, ny, nz, float(a), int(iters), _ptr(x), _ptr(y), _ptr(dots))
    return x, y, dots


# ---- FEM -------------------------------------------
def fem_ke(E: float = 1.0, nu: float = 0.3):
    ke = np.zeros((24, 24), dtype=np.float64)
    lib().or_fem_ke(float(E), float(nu), _ptr(ke))
    return ke


def fem_apply(u, E=1.0, nu=0.3, mask=None, dirichlet_z0=True):
    """u: [3][z][y][x] -> K u (Dirichlet identity rows/cols at z = 0)."""
    u = _f64(u)
    _, nz, ny, nx = u.shape
    ke = fem_ke(E, nu)
    y = np.empty_like(u)
    m = None if mask is None else np.ascontiguousarray(mask, dtype=np.uint8)
    lib().or_fem_apply(nx, ny, nz, _ptr(ke), None if m is None else _ptr(m),
                       int(bool(dirichlet_z0)), _ptr(u), _ptr(y))
    return y


def fem_rhs(dims, pressure=1.0, mask=None, dirichlet_z0=True):
    nx, ny, nz = dims
    b = np.zeros((3, nz, ny, nx), dtype=np.float64)
    m = None if mask is None else np.ascontiguousarray(mask, dtype=np.uint8)
    lib().or_fem_rhs(nx, ny, nz, None if m is None else _ptr(m), int(bool(dirichlet_z0)),
                     float(pressure), _ptr(b))
    return b


# ---- CG -----------------------------------
OP_LAPLACE7, OP_SPARSE7, OP_FEM27 = 0, 1, 2


def cg(b, x0=None, max_iter=100, rtol=0.0, op=OP_LAPLACE7, mask=None, E=1.0, nu=0.3):
    """Returns (x, CGResult, rr_history[iters+1])."""
    b = _f64(b)
    if op == OP_FEM27:
        _, nz, ny, nx = b.shape
    else:
        nz, ny, nx = b.shape
    x = np.zeros_like(b) if x0 is None else _f64(x0).copy()
    res = CGResult()
    hist = np.zeros(max_iter + 1, dtype=np.float64)
    ke = fem_ke(E, nu) if op == OP_FEM27 else None
    m = None if mask is None else np.ascontiguousarray(mask, dtype=np.uint8)
    rc = lib().or_cg(op, nx, ny, nz, None if m is None else _ptr(m),
                     None if ke is None else _ptr(ke), _ptr(b), _ptr(x), int(max_iter),
                     float(rtol), _ptr(hist), C.byref(res))
    if rc != 0:
        raise MemoryError("oracle CG allocation failed")
    return x, res, hist[: res.iters + 1]


# ---- D3Q19 LBM ---------------------------------------
def lbm_lattice():
    c = np.zeros((19, 3), dtype=np.int32)
    w = np.zeros(19, dtype=np.float64)
    opp = np.zeros(19, dtype=np.int32)
    lib().or_lbm_lattice(_ptr(c), _ptr(w), _ptr(opp))
    return c, w, opp


LBM_CAVITY, LBM_PERIODIC = 0, 1


def lbm_step(fin, omega, u_lid=0.05, rho_w=1.0, bc=LBM_CAVITY, active=None):
    """fin: [19][z][y][x] (any float dtype; computed in fp64) -> fout fp64.
    active: optional [z][y][x] mask of fluid cells (element-sparse domain,
    bounce-back at inactive sources; inactive cells -> 0)."""
    fin = _f64(fin)
    _, nz, ny, nx = fin.shape
    fout = np.empty_like(fin)
    if active is None:
        lib().or_lbm_step(nx, ny, nz, int(bc), float(omega), float(u_lid), float(rho_w),
                          _ptr(fin), _ptr(fout))
    else:
        m = np.ascontiguousarray(active, dtype=np.uint8)
        assert m.shape == (nz, ny, nx)
        lib().or_lbm_step_masked(nx, ny, nz, int(bc), float(omega), float(u_lid), float(rho_w),
                                 m.ctypes.data_as(C.c_void_p), _ptr(fin), _ptr(fout))
    return fout


def lbm_macroscopic(f):
    f = _f64(f)
    _, nz, ny, nx = f.shape
    rho = np.empty((nz, ny, nx), dtype=np.float64)
    u = np.empty((3, nz, ny, nx), dtype=np.float64)
    lib().or_lbm_macroscopic(nx, ny, nz, _ptr(f), _ptr(rho), _ptr(u))
    return rho, u


def lbm_omega(nx: int, u_lid: float = 0.05, re: float = 100.0) -> float:
    """Cavity parameters (SURVEY.md §8(c) c6 reading): nu = u_lid*Nx/Re,
    omega = 1/(3 nu + 1/2)."""
    nu = u_lid * nx / re
    return 1.0 / (3.0 * nu + 0.5)


# ---- D2Q9 Karman vortex street (readings in DESIGN.md §3)
D2Q9_CHANNEL, D2Q9_PERIODIC = 0, 1


def d2q9_lattice():
    c = np.zeros(18, dtype=np.int32)
    w = np.zeros(9, dtype=np.float64)
    o = np.zeros(9, dtype=np.int32)
    lib().or_d2q9_lattice(c.ctypes.data_as(C.c_void_p), w.ctypes.data_as(C.c_void_p), o.ctypes.data_as(C.c_void_p))
    return c.reshape(9, 2), w, o


def d2q9_step(fin, omega, u_in, cyl, bc=D2Q9_CHANNEL):
    """fin: [9][y][x] -> fout fp64 (computed in fp64 from the given values);
    cyl = (cx, cy, r) integers (r < 0: no cylinder)."""
    fin = _f64(fin)
    _, ny, nx = fin.shape
    fout = np.empty_like(fin)
    cx, cy, r = (int(v) for v in cyl)
    lib().or_d2q9_step(nx, ny, int(bc), float(omega), float(u_in), cx, cy, r, _ptr(fin), _ptr(fout))
    return fout
