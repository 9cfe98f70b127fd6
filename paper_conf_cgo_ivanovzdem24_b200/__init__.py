"""paper_conf_cgo_ivanovzdem24_b200 -- granularity-parameterised Rodinia kernels on B200.

Thin Python binding over the C ABI of ``librodinia_gran.so`` (``include/rodinia_gran.h``).
Argument marshalling only: every step of every workload runs in the library's sm_100a
kernels.  PyTorch supplies device memory (tensors), the current CUDA stream and process
groups; nothing here computes.  If the shared library is missing the import fails loudly:
there is no CPU or PyTorch fallback.

The functions carry the C names (``rodinia_hotspot`` ...) and take torch tensors.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("RODINIA_GRAN_LIB") or os.path.join(_HERE, "librodinia_gran.so")  # env: dev A/B builds

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build it with `python tools/build_lib.py` "
        "(or __graft_entry__.build()); there is no fallback implementation")

lib = ctypes.CDLL(LIB_PATH)

# ----------------------------------------------------------------------------- status codes
RODINIA_OK = 0
RODINIA_E_INVALID = -1
RODINIA_E_ILLEGAL_FACTOR = -2
RODINIA_E_SMEM = -3
RODINIA_E_FILTERED = -4
RODINIA_E_NOT_BUILT = -5
RODINIA_E_DEGENERATE = -6
RODINIA_E_NODEV = -7
RODINIA_E_CUDA = -8
RODINIA_E_NCCL = -9
RODINIA_E_NOMEM = -10
RODINIA_E_PRUNED = -11

RODINIA_FAITHFUL = 1
RODINIA_STREAM = 2
RODINIA_FORCE = 4  # run an instantiation the compile-time filter pruned (else RODINIA_E_FILTERED)

RODINIA_HOTSPOT, RODINIA_SRAD, RODINIA_PATHFINDER, RODINIA_LUD, RODINIA_HOTSPOT3D = 0, 1, 2, 3, 4
KERNELS = {"hotspot": 0, "srad": 1, "pathfinder": 2, "lud": 3, "hotspot3d": 4}


class RodiniaError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{status_string(status)}: {msg}")
        self.status = status


# ----------------------------------------------------------------------------- structs
class Granularity(ctypes.Structure):
    """rodinia_granularity: thread factor (x,y), block factor (x,y), temporal depth,
    index mode (0 coalescing-friendly / 1 contiguous) and flags."""
    _fields_ = [("thread_x", ctypes.c_int32), ("thread_y", ctypes.c_int32),
                ("block_x", ctypes.c_int32), ("block_y", ctypes.c_int32),
                ("temporal", ctypes.c_int32), ("index_mode", ctypes.c_int32),
                ("flags", ctypes.c_int32)]

    def astuple(self):
        return (self.thread_x, self.thread_y, self.block_x, self.block_y, self.temporal,
                self.index_mode, self.flags)

    def __repr__(self):
        return "Granularity(t=(%d,%d), b=(%d,%d), h=%d, mode=%d, flags=%d)" % self.astuple()


def gran(thread_x=1, thread_y=1, block_x=1, block_y=1, temporal=1, index_mode=0, flags=0):
    return Granularity(thread_x, thread_y, block_x, block_y, temporal, index_mode, flags)


UNCOARSENED = (1, 1, 1, 1, 1, 0, 0)


class HotspotCoeffs(ctypes.Structure):
    _fields_ = [("k", ctypes.c_float), ("rx", ctypes.c_float), ("ry", ctypes.c_float),
                ("rz", ctypes.c_float), ("amb", ctypes.c_float)]


class Problem(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_int64), ("cols", ctypes.c_int64),
                ("iterations", ctypes.c_int32), ("nranks", ctypes.c_int32),
                ("depth", ctypes.c_int32), ("reserved", ctypes.c_int32)]


class Hotspot3dCoeffs(ctypes.Structure):
    _fields_ = [(k, ctypes.c_float) for k in ("cc", "cw", "ce", "cs", "cn", "cb", "ct", "sdc", "amb")]


class TuneRow(ctypes.Structure):
    _fields_ = [("g", Granularity), ("median_ms", ctypes.c_float), ("regs", ctypes.c_int32),
                ("spill_bytes", ctypes.c_int32), ("smem_bytes", ctypes.c_int32),
                ("threads", ctypes.c_int32), ("ctas_per_sm", ctypes.c_int32),
                ("status", ctypes.c_int32), ("model_ms", ctypes.c_float)]

    def asdict(self):
        return dict(g=self.g.astuple(), median_ms=self.median_ms, regs=self.regs,
                    spill_bytes=self.spill_bytes, smem_bytes=self.smem_bytes,
                    threads=self.threads, ctas_per_sm=self.ctas_per_sm, status=self.status,
                    model_ms=self.model_ms)


# ----------------------------------------------------------------------------- signatures
_i32, _i64, _f32, _f64, _vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_float, ctypes.c_double, ctypes.c_void_p
_PG = ctypes.POINTER(Granularity)
_PC = ctypes.POINTER(HotspotCoeffs)

_SIGS = {
    "rodinia_last_error": ([], ctypes.c_char_p),
    "rodinia_status_string": ([_i32], ctypes.c_char_p),
    "rodinia_sync": ([_vp], _i32),
    "rodinia_abi_version": ([], _i32),
    "rodinia_launch_count": ([], _i64),
    "rodinia_kernel_timing": ([_i32], _i32),
    "rodinia_kernel_time": ([ctypes.POINTER(_f64), ctypes.POINTER(_i64)], _i32),
    "rodinia_hotspot_coeffs_rodinia": ([_i64, _i64, _f64, _f64, _PC], _i32),
    "rodinia_hotspot": ([_vp, _vp, _vp, _vp, _i64, _i64, _i32, _PC, _PG, _vp], _i32),
    "rodinia_hotspot_host": ([_vp, _vp, _vp, _i64, _i64, _i32, _PC, _PG, _vp], _i32),
    "rodinia_hotspot_host_batch": ([ctypes.POINTER(_vp), ctypes.POINTER(_vp), ctypes.POINTER(_vp), _i32, _i64, _i64,
                                    _i32, _PC, _PG, _vp], _i32),
    "rodinia_hotspot3d_coeffs_rodinia": ([_i64, _i64, _i64, _f64, _f64, _f64, ctypes.c_void_p], _i32),
    "rodinia_hotspot3d": ([_vp, _vp, _vp, _vp, _i64, _i64, _i64, _i32, _vp, _PG, _vp], _i32),
    "rodinia_hotspot3d_host": ([_vp, _vp, _vp, _i64, _i64, _i64, _i32, _vp, _PG, _vp], _i32),
    "rodinia_srad": ([_vp, _i64, _i64, _i64, _i64, _i64, _i64, _f32, _i32, _PG, _vp], _i32),
    "rodinia_srad_host": ([_vp, _i64, _i64, _i64, _i64, _i64, _i64, _f32, _i32, _PG, _vp], _i32),
    "rodinia_srad_v1": ([_vp, _i64, _i64, _f32, _i32, _PG, _vp], _i32),
    "rodinia_srad_v1_host": ([_vp, _i64, _i64, _f32, _i32, _PG, _vp], _i32),
    "rodinia_pathfinder": ([_vp, _i64, _i64, _vp, _PG, _vp], _i32),
    "rodinia_pathfinder_host": ([_vp, _i64, _i64, _vp, _PG, _vp], _i32),
    "rodinia_lud": ([_vp, _i64, _i32, _PG, _vp], _i32),
    "rodinia_lud_host": ([_vp, _i64, _i32, _PG, _vp], _i32),
    "rodinia_variants": ([_i32, ctypes.POINTER(TuneRow), ctypes.POINTER(_i32)], _i32),
    "rodinia_tune": ([_i32, ctypes.POINTER(Problem), _i32, _PG, ctypes.POINTER(TuneRow),
                      ctypes.POINTER(_i32)], _i32),
    "rodinia_tune_pruned": ([_i32, ctypes.POINTER(Problem), _i32, _i32, _PG, ctypes.POINTER(TuneRow),
                             ctypes.POINTER(_i32)], _i32),
    "rodinia_model_ms": ([_i32, ctypes.POINTER(Problem), ctypes.POINTER(TuneRow)], _i32),
    "rodinia_resolve": ([_i32, ctypes.POINTER(Problem), _PG], _i32),
    "rodinia_split_total": ([_i32, _i32, ctypes.POINTER(_i32)], _i32),
    "rodinia_slab": ([_i64, _i32, _i32, ctypes.POINTER(_i64), ctypes.POINTER(_i64)], _i32),
    "rodinia_comm_unique_id": ([ctypes.c_char_p], _i32),
    "rodinia_comm_init": ([ctypes.POINTER(_vp), _i32, _i32, ctypes.c_char_p], _i32),
    "rodinia_comm_init_local": ([ctypes.POINTER(_vp), _i32], _i32),
    "rodinia_comm_destroy": ([_vp], _i32),
    "rodinia_hotspot_dist": ([_vp, _vp, _vp, _vp, _i64, _i64, _i32, _PC, _PG, _vp], _i32),
    "rodinia_srad_dist": ([_vp, _vp, _i64, _i64, _i64, _i64, _i64, _i64, _f32, _i32, _PG, _vp], _i32),
    "rodinia_lud_dist": ([_vp, _vp, _i64, _i32, _i32, _vp], _i32),
    "rodinia_lud_dist_layout": ([_i64, _i32, _i32, _i32, ctypes.POINTER(_i64), ctypes.POINTER(_i64)], _i32),
    "rodinia_dist_schedule": ([_i32, _i64, _i64, _i32, _i32, _i32, _i64, _i64, _i64, _i64, _PG, _vp], _i32),
}

EXPORTED = sorted(_SIGS)
_missing = []
for _name, (_args, _res) in _SIGS.items():
    _f = getattr(lib, _name, None)
    if _f is None:
        _missing.append(_name)
        continue
    _f.argtypes = _args
    _f.restype = _res


def status_string(s: int) -> str:
    return lib.rodinia_status_string(s).decode()


def last_error() -> str:
    return lib.rodinia_last_error().decode()


def check(status: int, what: str = ""):
    if status != RODINIA_OK:
        raise RodiniaError(status, f"{what}: {last_error()}")


def _g(g) -> "ctypes.pointer | None":
    if g is None:
        return None
    if isinstance(g, Granularity):
        return ctypes.pointer(g)
    if isinstance(g, dict):
        return ctypes.pointer(gran(**g))
    return ctypes.pointer(Granularity(*g))


def _stream(stream):
    if stream is None:
        import torch
        return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return ctypes.c_void_p(stream)
    return ctypes.c_void_p(stream.cuda_stream)


def _dev(t, dtype, name):
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    return ctypes.c_void_p(t.data_ptr())


# ----------------------------------------------------------------------------- hotspot
def rodinia_hotspot_coeffs_rodinia(rows: int, cols: int, chip_w: float = 0.016,
                                   chip_h: float = 0.016) -> HotspotCoeffs:
    c = HotspotCoeffs()
    check(lib.rodinia_hotspot_coeffs_rodinia(rows, cols, chip_w, chip_h, ctypes.byref(c)),
          "rodinia_hotspot_coeffs_rodinia")
    return c


def coeffs(k, rx, ry, rz, amb=80.0) -> HotspotCoeffs:
    return HotspotCoeffs(k, rx, ry, rz, amb)


def rodinia_hotspot(temp, power, iterations: int, coeffs=None, g=None, out=None, scratch=None,
                    stream=None):
    """`iterations` hotspot steps of temp (R x C float32 CUDA tensor); returns temp_out."""
    import torch
    if temp.dim() != 2 or power.shape != temp.shape:
        raise ValueError("temp and power must be equal-shaped 2-D tensors")
    R, C = temp.shape
    if out is None:
        out = torch.empty_like(temp)
    st = lib.rodinia_hotspot(
        _dev(temp, torch.float32, "temp"), _dev(power, torch.float32, "power"),
        _dev(out, torch.float32, "out"),
        None if scratch is None else _dev(scratch, torch.float32, "scratch"),
        R, C, int(iterations), None if coeffs is None else ctypes.byref(coeffs), _g(g),
        _stream(stream))
    check(st, "rodinia_hotspot")
    return out


def rodinia_hotspot_host_batch(temps, powers, iterations: int, coeffs=None, g=None, outs=None, stream=None):
    """Batch of independent problems with host buffers (numpy float32, ideally pinned): copies
    of neighbouring problems overlap the solves (two device buffer sets).  Returns the outputs."""
    import numpy as np
    ts = [np.ascontiguousarray(t, dtype=np.float32) for t in temps]
    ps = [np.ascontiguousarray(p, dtype=np.float32) for p in powers]
    if len(ts) != len(ps) or not ts:
        raise ValueError("temps and powers must be non-empty lists of equal length")
    R, C = ts[0].shape
    if any(t.shape != (R, C) for t in ts + ps):
        raise ValueError("all problems must have the same shape")
    if outs is None:
        outs = [np.empty_like(ts[0]) for _ in ts]
    n = len(ts)
    arr = lambda xs: (_vp * n)(*[x.ctypes.data for x in xs])
    st = lib.rodinia_hotspot_host_batch(arr(ts), arr(ps), arr(outs), n, R, C, int(iterations),
                                        None if coeffs is None else ctypes.byref(coeffs), _g(g), _stream(stream))
    check(st, "rodinia_hotspot_host_batch")
    return outs


def rodinia_hotspot_host(temp, power, iterations: int, coeffs=None, g=None, out=None,
                         stream=None):
    """Host-buffer variant: numpy float32 / CPU tensors in, H2D + solve + D2H inside the call."""
    import numpy as np
    t = np.ascontiguousarray(temp, dtype=np.float32)
    p = np.ascontiguousarray(power, dtype=np.float32)
    if out is None:
        out = np.empty_like(t)
    R, C = t.shape
    st = lib.rodinia_hotspot_host(
        ctypes.c_void_p(t.ctypes.data), ctypes.c_void_p(p.ctypes.data),
        ctypes.c_void_p(out.ctypes.data), R, C, int(iterations),
        None if coeffs is None else ctypes.byref(coeffs), _g(g), _stream(stream))
    check(st, "rodinia_hotspot_host")
    return out


# ----------------------------------------------------------------------------- hotspot3d
def rodinia_hotspot3d_coeffs_rodinia(nx: int, ny: int, nz: int, chip_w: float = 0.016, chip_h: float = 0.016,
                                     t_chip: float = 0.0005) -> Hotspot3dCoeffs:
    c = Hotspot3dCoeffs()
    check(lib.rodinia_hotspot3d_coeffs_rodinia(nx, ny, nz, chip_w, chip_h, t_chip, ctypes.addressof(c)),
          "rodinia_hotspot3d_coeffs_rodinia")
    return c


def rodinia_hotspot3d(temp, power, iterations: int, coeffs=None, g=None, out=None, scratch=None, stream=None):
    """`iterations` hotspot3D steps of temp ((nz, ny, nx) float32 CUDA tensor); returns temp_out."""
    import torch
    if temp.dim() != 3 or power.shape != temp.shape:
        raise ValueError("temp and power must be equal-shaped (nz, ny, nx) tensors")
    nz, ny, nx = temp.shape
    if out is None:
        out = torch.empty_like(temp)
    check(lib.rodinia_hotspot3d(_dev(temp, torch.float32, "temp"), _dev(power, torch.float32, "power"),
                                _dev(out, torch.float32, "out"),
                                None if scratch is None else _dev(scratch, torch.float32, "scratch"),
                                nx, ny, nz, int(iterations), None if coeffs is None else ctypes.addressof(coeffs),
                                _g(g), _stream(stream)), "rodinia_hotspot3d")
    return out


def rodinia_hotspot3d_host(temp, power, iterations: int, coeffs=None, g=None, stream=None):
    import numpy as np
    t = np.ascontiguousarray(temp, dtype=np.float32)
    p = np.ascontiguousarray(power, dtype=np.float32)
    out = np.empty_like(t)
    nz, ny, nx = t.shape
    check(lib.rodinia_hotspot3d_host(ctypes.c_void_p(t.ctypes.data), ctypes.c_void_p(p.ctypes.data),
                                     ctypes.c_void_p(out.ctypes.data), nx, ny, nz, int(iterations),
                                     None if coeffs is None else ctypes.addressof(coeffs), _g(g), _stream(stream)),
          "rodinia_hotspot3d_host")
    return out


# ----------------------------------------------------------------------------- srad
def rodinia_srad(J, r1, r2, c1, c2, lam: float, niter: int, g=None, stream=None):
    """niter srad_v2 iterations on J (R x C float32 CUDA tensor, in place); returns J."""
    import torch
    R, C = J.shape
    check(lib.rodinia_srad(_dev(J, torch.float32, "J"), R, C, r1, r2, c1, c2, float(lam),
                           int(niter), _g(g), _stream(stream)), "rodinia_srad")
    return J


def rodinia_srad_host(J, r1, r2, c1, c2, lam: float, niter: int, g=None, stream=None):
    import numpy as np
    a = np.ascontiguousarray(J, dtype=np.float32).copy()
    R, C = a.shape
    check(lib.rodinia_srad_host(ctypes.c_void_p(a.ctypes.data), R, C, r1, r2, c1, c2, float(lam),
                                int(niter), _g(g), _stream(stream)), "rodinia_srad_host")
    return a


def rodinia_srad_v1(image, lam: float, niter: int, g=None, stream=None):
    """Rodinia srad_v1 on image (R x C float32 CUDA tensor, pixel values 0..255, in place)."""
    import torch
    R, C = image.shape
    check(lib.rodinia_srad_v1(_dev(image, torch.float32, "image"), R, C, float(lam), int(niter), _g(g),
                              _stream(stream)), "rodinia_srad_v1")
    return image


def rodinia_srad_v1_host(image, lam: float, niter: int, g=None, stream=None):
    import numpy as np
    a = np.ascontiguousarray(image, dtype=np.float32).copy()
    R, C = a.shape
    check(lib.rodinia_srad_v1_host(ctypes.c_void_p(a.ctypes.data), R, C, float(lam), int(niter), _g(g),
                                   _stream(stream)), "rodinia_srad_v1_host")
    return a


# ----------------------------------------------------------------------------- pathfinder
def rodinia_pathfinder(wall, g=None, out=None, stream=None):
    import torch
    R, C = wall.shape
    if out is None:
        out = torch.empty(C, dtype=torch.int32, device=wall.device)
    check(lib.rodinia_pathfinder(_dev(wall, torch.int32, "wall"), R, C,
                                 _dev(out, torch.int32, "out"), _g(g), _stream(stream)),
          "rodinia_pathfinder")
    return out


def rodinia_pathfinder_host(wall, g=None, stream=None):
    import numpy as np
    w = np.ascontiguousarray(wall, dtype=np.int32)
    out = np.empty(w.shape[1], dtype=np.int32)
    check(lib.rodinia_pathfinder_host(ctypes.c_void_p(w.ctypes.data), w.shape[0], w.shape[1],
                                      ctypes.c_void_p(out.ctypes.data), _g(g), _stream(stream)),
          "rodinia_pathfinder_host")
    return out


# ----------------------------------------------------------------------------- lud
def rodinia_lud(a, panel: int = 16, g=None, stream=None):
    """In-place blocked LU of a (n x n float32 CUDA tensor); returns a (packed L\\U)."""
    import torch
    n = a.shape[0]
    if a.dim() != 2 or a.shape[1] != n:
        raise ValueError("lud needs a square matrix")
    check(lib.rodinia_lud(_dev(a, torch.float32, "a"), n, int(panel), _g(g), _stream(stream)),
          "rodinia_lud")
    return a


def rodinia_lud_host(a, panel: int = 16, g=None, stream=None):
    import numpy as np
    m = np.ascontiguousarray(a, dtype=np.float32).copy()
    check(lib.rodinia_lud_host(ctypes.c_void_p(m.ctypes.data), m.shape[0], int(panel), _g(g),
                               _stream(stream)), "rodinia_lud_host")
    return m


# ----------------------------------------------------------------------------- variants / tune
def _kernel(k):
    return KERNELS[k] if isinstance(k, str) else int(k)


def rodinia_variants(kernel):
    n = _i32(0)
    check(lib.rodinia_variants(_kernel(kernel), None, ctypes.byref(n)), "rodinia_variants")
    rows = (TuneRow * max(n.value, 1))()
    check(lib.rodinia_variants(_kernel(kernel), rows, ctypes.byref(n)), "rodinia_variants")
    return [rows[i].asdict() for i in range(n.value)]


def rodinia_tune(kernel, rows: int, cols: int, iterations: int = 1, nranks: int = 1, reps: int = 3,
                 depth: int = 0):
    """Timing-driven selection. Returns (best Granularity, [row dicts])."""
    p = Problem(rows, cols, iterations, nranks, depth, 0)
    best = Granularity()
    cap = _i32(4096)
    out = (TuneRow * cap.value)()
    check(lib.rodinia_tune(_kernel(kernel), ctypes.byref(p), reps, ctypes.byref(best), out,
                           ctypes.byref(cap)), "rodinia_tune")
    return best, [out[i].asdict() for i in range(min(cap.value, 4096))]


def rodinia_tune_pruned(kernel, rows: int, cols: int, iterations: int = 1, keep: int = 8, nranks: int = 1,
                        reps: int = 3, depth: int = 0):
    """Timing-driven selection after heuristic pre-pruning:
    only the `keep` candidates the kernel-statistics model ranks best are timed."""
    p = Problem(rows, cols, iterations, nranks, depth, 0)
    best = Granularity()
    cap = _i32(4096)
    out = (TuneRow * cap.value)()
    check(lib.rodinia_tune_pruned(_kernel(kernel), ctypes.byref(p), reps, keep, ctypes.byref(best), out,
                                  ctypes.byref(cap)), "rodinia_tune_pruned")
    return best, [out[i].asdict() for i in range(min(cap.value, 4096))]


def rodinia_model_ms(kernel, g, rows: int, cols: int, iterations: int = 1, depth: int = 0, regs: int = -1,
                     threads: int = 0, smem_bytes: int = 0, ctas_per_sm: int = 0, spill_bytes: int = 0) -> float:
    """The pre-pruning model's estimate (ms) of one call at granularity g; -1 if not modelled."""
    p = Problem(rows, cols, iterations, 1, depth, 0)
    r = TuneRow()
    r.g = g if isinstance(g, Granularity) else gran(*g) if isinstance(g, (tuple, list)) else gran(**g)
    r.regs, r.threads, r.smem_bytes, r.ctas_per_sm, r.spill_bytes = regs, threads, smem_bytes, ctas_per_sm, spill_bytes
    check(lib.rodinia_model_ms(_kernel(kernel), ctypes.byref(p), ctypes.byref(r)), "rodinia_model_ms")
    return float(r.model_ms)


def rodinia_resolve(kernel, rows: int, cols: int, iterations: int = 1, nranks: int = 1, depth: int = 0):
    p = Problem(rows, cols, iterations, nranks, depth, 0)
    g = Granularity()
    check(lib.rodinia_resolve(_kernel(kernel), ctypes.byref(p), ctypes.byref(g)), "rodinia_resolve")
    return g


def rodinia_split_total(total: int, ndims: int = 3):
    """Balance a total coarsening factor over ndims dimensions (footnote 4)."""
    out = (_i32 * 3)()
    check(lib.rodinia_split_total(int(total), int(ndims), out), "rodinia_split_total")
    return tuple(out[:ndims])


def rodinia_sync(stream=None):
    check(lib.rodinia_sync(_stream(stream)), "rodinia_sync")


def rodinia_launch_count() -> int:
    return int(lib.rodinia_launch_count())


def rodinia_kernel_timing(enable: bool) -> None:
    """Start (clearing earlier records) or stop event timing of the stepping launches."""
    check(lib.rodinia_kernel_timing(1 if enable else 0), "rodinia_kernel_timing")


def rodinia_kernel_time():
    """(summed milliseconds, number of timed launches) since the last enable."""
    ms, n = _f64(0.0), _i64(0)
    check(lib.rodinia_kernel_time(ctypes.byref(ms), ctypes.byref(n)), "rodinia_kernel_time")
    return float(ms.value), int(n.value)


# ----------------------------------------------------------------------------- multi-GPU
def rodinia_slab(global_rows: int, nranks: int, rank: int):
    r0, n = _i64(0), _i64(0)
    check(lib.rodinia_slab(global_rows, nranks, rank, ctypes.byref(r0), ctypes.byref(n)),
          "rodinia_slab")
    return r0.value, n.value



from . import dist  # noqa: E402  (row-slab multi-GPU layer)
