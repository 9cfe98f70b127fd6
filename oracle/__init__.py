"""CPU oracle (TEST INFRASTRUCTURE ONLY).

Thin ctypes wrapper over ``oracle/rodinia_oracle.c`` (plain C, fp64, single thread).
Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
``paper_conf_cgo_ivanovzdem24_b200`` never imports it and shares no code with it.

Each function cites the Rodinia kernel whose plain definition the C code writes out (the
paper transforms existing Rodinia v3 kernels without changing their results, PAPER.md:145,
PAPER.md:295); every reading where the paper is silent is listed in DESIGN.md §3.

Parity status: every function here is pinned by ``tests/test_oracle_*.py`` against closed
forms, brute force, library routines or hand-checked fixtures (DESIGN.md §4 lists the pin
for each function).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "rodinia_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_LIB_OMP = os.path.join(_HERE, "liboracle_omp.so")
_lock = threading.Lock()
_lib = None
_threads = 1

OK = 0
EINVAL = -1
EDEGENERATE = -6
ENOMEM = -10

_CFLAGS = ["-O2", "-std=c99", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]


def build(force: bool = False, omp: bool = False) -> str:
    """Compile liboracle.so with gcc (no fast-math, no FMA contraction); with omp=True the
    OpenMP build liboracle_omp.so (same source, per-cell stencil loops threaded, identical bits).
    """
    lib = _LIB_OMP if omp else _LIB
    if force or not os.path.exists(lib) or os.path.getmtime(lib) < os.path.getmtime(_SRC):
        tmp = lib + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *_CFLAGS, *(["-fopenmp"] if omp else []), "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, lib)
    return lib


def set_threads(n: int) -> int:
    """Select the single-threaded build (n == 1, the default) or the OpenMP build with n threads
    (n == 0: all host cores, os.cpu_count()).  Returns the thread count in effect.  Results are
    bitwise identical either way (only independent per-cell loops are threaded)."""
    global _lib, _threads
    n = os.cpu_count() or 1 if n == 0 else int(n)
    with _lock:
        if n != _threads or _lib is None:
            _lib = None
            _threads = n
    lib = _load()
    return int(lib.oracle_set_threads(n))


def threads() -> int:
    return _threads


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build(omp=_threads > 1))
            lib.oracle_set_threads.argtypes = [ctypes.c_int]
            lib.oracle_set_threads.restype = ctypes.c_int
            d, l, i = ctypes.c_double, ctypes.c_long, ctypes.c_int
            pd = ctypes.POINTER(ctypes.c_double)
            pi32 = ctypes.POINTER(ctypes.c_int32)
            lib.oracle_hotspot_coeffs_rodinia.argtypes = [l, l, d, d, pd]
            lib.oracle_hotspot.argtypes = [pd, pd, pd, l, l, i, d, d, d, d, d]
            lib.oracle_srad_q0sqr.argtypes = [pd, l, l, l, l, l, l, pd]
            lib.oracle_srad_coeff.argtypes = [pd, l, l, d, pd]
            lib.oracle_srad_step.argtypes = [pd, l, l, d, d]
            lib.oracle_srad.argtypes = [pd, l, l, l, l, l, l, d, i, pd]
            lib.oracle_pathfinder.argtypes = [pi32, l, l, pi32]
            lib.oracle_lud.argtypes = [pd, l]
            lib.oracle_srad_v1.argtypes = [pd, l, l, d, i]
            for f in ("oracle_hotspot_coeffs_rodinia", "oracle_hotspot", "oracle_srad_q0sqr",
                      "oracle_srad_coeff", "oracle_srad_step", "oracle_srad",
                      "oracle_pathfinder", "oracle_lud", "oracle_srad_v1"):
                getattr(lib, f).restype = ctypes.c_int
            _lib = lib
    return _lib


class OracleError(RuntimeError):
    def __init__(self, code: int, what: str):
        super().__init__(f"{what}: oracle status {code}")
        self.code = code


def _chk(code: int, what: str):
    if code != OK:
        raise OracleError(code, what)


def _f64(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.float64))


def _p(a: np.ndarray, t=ctypes.c_double):
    return a.ctypes.data_as(ctypes.POINTER(t))


# --------------------------------------------------------------------------- hotspot
def hotspot_coeffs_rodinia(rows: int, cols: int, chip_w: float = 0.016, chip_h: float = 0.016):
    """Rodinia hotspot chip constants -> dict(k, rx, ry, rz, amb) in fp64 (H1)."""
    out = np.zeros(5, dtype=np.float64)
    _chk(_load().oracle_hotspot_coeffs_rodinia(rows, cols, chip_w, chip_h, _p(out)), "coeffs")
    return dict(k=out[0], rx=out[1], ry=out[2], rz=out[3], amb=out[4])


def hotspot(t0, power, iterations: int, k, rx, ry, rz, amb=80.0) -> np.ndarray:
    """`iterations` Jacobi steps of Rodinia hotspot `calculate_temp` (h = 1), fp64."""
    t0 = _f64(t0)
    p = _f64(power)
    if t0.ndim != 2 or p.shape != t0.shape:
        raise ValueError("t0 and power must be equal-shaped 2-D arrays")
    out = np.empty_like(t0)
    R, C = t0.shape
    _chk(_load().oracle_hotspot(_p(t0), _p(p), _p(out), R, C, int(iterations),
                                float(k), float(rx), float(ry), float(rz), float(amb)), "hotspot")
    return out


# --------------------------------------------------------------------------- srad
def srad_q0sqr(J, r1, r2, c1, c2) -> float:
    J = _f64(J)
    R, C = J.shape
    q = ctypes.c_double(0.0)
    _chk(_load().oracle_srad_q0sqr(_p(J), R, C, r1, r2, c1, c2, ctypes.byref(q)), "q0sqr")
    return q.value


def srad_coeff(J, q0sqr: float) -> np.ndarray:
    """Pass 1 (srad_cuda_1): diffusion coefficient c for every cell."""
    J = _f64(J)
    c = np.empty_like(J)
    R, C = J.shape
    _chk(_load().oracle_srad_coeff(_p(J), R, C, float(q0sqr), _p(c)), "srad_coeff")
    return c


def srad_step(J, q0sqr: float, lam: float) -> np.ndarray:
    J = _f64(J).copy()
    R, C = J.shape
    _chk(_load().oracle_srad_step(_p(J), R, C, float(q0sqr), float(lam)), "srad_step")
    return J


def srad(J, r1, r2, c1, c2, lam: float, niter: int, return_q0: bool = False):
    """niter srad_v2 iterations (ROI stats in fp64, pass 1, pass 2), fp64."""
    J = _f64(J).copy()
    R, C = J.shape
    q0 = np.zeros(max(niter, 1), dtype=np.float64)
    _chk(_load().oracle_srad(_p(J), R, C, r1, r2, c1, c2, float(lam), int(niter), _p(q0)), "srad")
    return (J, q0[:niter]) if return_q0 else J


def srad_v1(image, lam: float, niter: int):
    """Rodinia srad_v1: extract (exp(x/255)), niter iterations with whole-image statistics,
    compress (log(J)*255); fp64."""
    a = _f64(image).copy()
    R, C = a.shape
    _chk(_load().oracle_srad_v1(_p(a), R, C, float(lam), int(niter)), "srad_v1")
    return a


# --------------------------------------------------------------------------- pathfinder
def pathfinder(wall) -> np.ndarray:
    w = np.ascontiguousarray(np.asarray(wall, dtype=np.int32))
    R, C = w.shape
    out = np.empty(C, dtype=np.int32)
    _chk(_load().oracle_pathfinder(_p(w, ctypes.c_int32), R, C, _p(out, ctypes.c_int32)),
         "pathfinder")
    return out


# --------------------------------------------------------------------------- lud
def lud(a) -> np.ndarray:
    """Doolittle LU without pivoting (fp64), packed: unit L below the diagonal, U on/above."""
    a = _f64(a).copy()
    if a.ndim != 2 or a.shape[0] != a.shape[1]:
        raise ValueError("lud needs a square matrix")
    _chk(_load().oracle_lud(_p(a), a.shape[0]), "lud")
    return a


def lud_unpack(packed: np.ndarray):
    """Split a packed LU into (L unit-lower, U upper)."""
    n = packed.shape[0]
    L = np.tril(packed, -1) + np.eye(n, dtype=packed.dtype)
    U = np.triu(packed)
    return L, U


# --------------------------------------------------------------------------- hotspot3D
def hotspot3d_coeffs(nx: int, ny: int, nz: int, chip_w: float = 0.016, chip_h: float = 0.016,
                     t_chip: float = 0.0005):
    """Rodinia hotspot3D constants -> dict(cc, cw, ce, cs, cn, cb, ct, sdc, amb), fp64."""
    lib = _load()
    lib.oracle_hotspot3d_coeffs.argtypes = [ctypes.c_long] * 3 + [ctypes.c_double] * 3 + [
        ctypes.POINTER(ctypes.c_double)]
    lib.oracle_hotspot3d_coeffs.restype = ctypes.c_int
    out = np.zeros(9, dtype=np.float64)
    _chk(lib.oracle_hotspot3d_coeffs(nx, ny, nz, chip_w, chip_h, t_chip, _p(out)), "hotspot3d_coeffs")
    return dict(zip(("cc", "cw", "ce", "cs", "cn", "cb", "ct", "sdc", "amb"), out.tolist()))


HS3D_KEYS = ("cc", "cw", "ce", "cs", "cn", "cb", "ct", "sdc", "amb")


def hotspot3d(t0, power, iterations: int, coef: dict) -> np.ndarray:
    """`iterations` Jacobi steps of Rodinia hotspot3D (7-point, clamped), fp64.  Arrays are
    (nz, ny, nx), x fastest."""
    lib = _load()
    pd = ctypes.POINTER(ctypes.c_double)
    lib.oracle_hotspot3d.argtypes = [pd, pd, pd, ctypes.c_long, ctypes.c_long, ctypes.c_long, ctypes.c_int, pd]
    lib.oracle_hotspot3d.restype = ctypes.c_int
    t0 = _f64(t0)
    p = _f64(power)
    if t0.ndim != 3 or p.shape != t0.shape:
        raise ValueError("t0 and power must be equal-shaped (nz, ny, nx) arrays")
    nz, ny, nx = t0.shape
    cf = np.array([coef[k] for k in HS3D_KEYS], dtype=np.float64)
    out = np.empty_like(t0)
    _chk(lib.oracle_hotspot3d(_p(t0), _p(p), _p(out), nx, ny, nz, int(iterations), _p(cf)), "hotspot3d")
    return out
