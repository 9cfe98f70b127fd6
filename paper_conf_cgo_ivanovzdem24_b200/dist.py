"""Row-slab multi-GPU layer (hotspot, srad): thin binding over rodinia_comm_* / *_dist.

One process per GPU.  `HaloComm.from_process_group()` bootstraps the library-owned NCCL
communicator from a torch.distributed process group (rank 0 creates the NCCL unique id,
broadcast_object_list ships it); the halo exchange itself runs inside the library
(ncclSend/ncclRecv on the compute stream).  `HaloComm.local(P)` keeps P slabs
on the current device (cudaMemcpyAsync halos) to exercise the same slab logic on one GPU.
"""
from __future__ import annotations

import ctypes
import os

from . import (HotspotCoeffs, _dev, _g, _stream, check, lib)


def _nccl_path():
    """Point the library at the libnccl.so.2 torch uses (never the system copy)."""
    if os.environ.get("RODINIA_NCCL_LIB"):
        return os.environ["RODINIA_NCCL_LIB"]
    try:
        import nvidia.nccl
        p = os.path.join(list(nvidia.nccl.__path__)[0], "lib", "libnccl.so.2")
        if os.path.exists(p):
            os.environ["RODINIA_NCCL_LIB"] = p
            return p
    except Exception:
        pass
    return None


def unique_id() -> bytes:
    _nccl_path()
    buf = ctypes.create_string_buffer(128)
    check(lib.rodinia_comm_unique_id(buf), "rodinia_comm_unique_id")
    return buf.raw


def slab(global_rows: int, nranks: int, rank: int):
    r0, n = ctypes.c_int64(0), ctypes.c_int64(0)
    check(lib.rodinia_slab(global_rows, nranks, rank, ctypes.byref(r0), ctypes.byref(n)), "rodinia_slab")
    return r0.value, n.value


class DistPlan(ctypes.Structure):
    """rodinia_dist_plan: the schedule one rank follows (rodinia_dist_schedule)."""
    _fields_ = [("row0", ctypes.c_int64), ("own", ctypes.c_int64), ("top", ctypes.c_int32),
                ("bot", ctypes.c_int32), ("period", ctypes.c_int32), ("send_up", ctypes.c_int32),
                ("send_down", ctypes.c_int32), ("exchanges", ctypes.c_int32), ("overlap", ctypes.c_int32),
                ("reserved", ctypes.c_int32), ("cone_r0", ctypes.c_int64), ("cone_r1", ctypes.c_int64),
                ("cone_c0", ctypes.c_int64), ("cone_c1", ctypes.c_int64)]

    def asdict(self):
        return {k: getattr(self, k) for k, _ in self._fields_ if k != "reserved"}


def schedule(kernel, global_rows: int, cols: int, nranks: int, rank: int, iterations: int,
             roi=(0, 0, 0, 0), g=None) -> dict:
    """Host-only: the slab, halo depths, exchange period/sizes and (srad) ROI-cone window the
    library uses for `rank` (no device needed)."""
    from . import _kernel
    out = DistPlan()
    r1, r2, c1, c2 = roi
    check(lib.rodinia_dist_schedule(_kernel(kernel), global_rows, cols, nranks, rank, int(iterations),
                                    r1, r2, c1, c2, _g(g), ctypes.byref(out)), "rodinia_dist_schedule")
    return out.asdict()


def lud_layout(n: int, prow: int, pcol: int, rank: int):
    """Host-only: (mloc, nloc), the local matrix shape of `rank` in rodinia_lud_dist's 2-D
    block-cyclic layout (NB = 128 blocks, rank = pr * pcol + pc)."""
    m, k = ctypes.c_int64(0), ctypes.c_int64(0)
    check(lib.rodinia_lud_dist_layout(n, prow, pcol, rank, ctypes.byref(m), ctypes.byref(k)),
          "rodinia_lud_dist_layout")
    return m.value, k.value


LUD_NB = 128


def _bc_index(n: int, P: int, p: int):
    """Global indices of the rows (or columns) of the blocks I = p (mod P), increasing I."""
    import numpy as np
    nb = (n + LUD_NB - 1) // LUD_NB
    return np.concatenate([np.arange(I * LUD_NB, min(n, (I + 1) * LUD_NB)) for I in range(p, nb, P)] or
                          [np.zeros(0, dtype=np.int64)])


def block_cyclic_scatter(A, prow: int, pcol: int):
    """Layout only: the prow*pcol local matrices of a global n x n tensor (rank order)."""
    import torch
    n = A.shape[0]
    out = []
    for r in range(prow * pcol):
        ri = torch.as_tensor(_bc_index(n, prow, r // pcol), device=A.device)
        ci = torch.as_tensor(_bc_index(n, pcol, r % pcol), device=A.device)
        out.append(A[ri][:, ci].contiguous())
    return out


def block_cyclic_gather(parts, n: int, prow: int, pcol: int):
    """Layout only: the global n x n tensor from the local matrices (rank order)."""
    import torch
    A = torch.empty((n, n), dtype=parts[0].dtype, device=parts[0].device)
    for r, x in enumerate(parts):
        ri = torch.as_tensor(_bc_index(n, prow, r // pcol), device=A.device)
        ci = torch.as_tensor(_bc_index(n, pcol, r % pcol), device=A.device)
        if len(ri) and len(ci):
            A[ri[:, None], ci[None, :]] = x
    return A


class HaloComm:
    def __init__(self, handle, nranks: int, rank: int, local: bool):
        self.handle = handle
        self.nranks = nranks
        self.rank = rank
        self.local = local

    @classmethod
    def from_process_group(cls, group=None):
        import torch.distributed as dist
        ws, rank = dist.get_world_size(group), dist.get_rank(group)
        obj = [unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0, group=group)
        h = ctypes.c_void_p()
        _nccl_path()
        check(lib.rodinia_comm_init(ctypes.byref(h), ws, rank, obj[0]), "rodinia_comm_init")
        return cls(h, ws, rank, local=False)

    @classmethod
    def local_slabs(cls, nranks: int):
        h = ctypes.c_void_p()
        check(lib.rodinia_comm_init_local(ctypes.byref(h), nranks), "rodinia_comm_init_local")
        return cls(h, nranks, 0, local=True)

    def close(self):
        if self.handle:
            check(lib.rodinia_comm_destroy(self.handle), "rodinia_comm_destroy")
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ------------------------------------------------------------------ marshalling
    def _ptrs(self, x, dtype, name):
        if self.local:
            arr = (ctypes.c_void_p * self.nranks)(*[_dev(t, dtype, name).value for t in x])
            return ctypes.cast(arr, ctypes.c_void_p), arr
        return _dev(x, dtype, name), None

    def hotspot(self, temp_local, power_local, out_local, global_rows: int, iterations: int,
                coeffs: HotspotCoeffs | None = None, g=None, stream=None):
        """One rank's slab (or, for a local communicator, lists of all slabs)."""
        import torch
        t, keep1 = self._ptrs(temp_local, torch.float32, "temp")
        p, keep2 = self._ptrs(power_local, torch.float32, "power")
        o, keep3 = self._ptrs(out_local, torch.float32, "out")
        cols = (temp_local[0] if self.local else temp_local).shape[1]
        check(lib.rodinia_hotspot_dist(self.handle, t, p, o, global_rows, cols, int(iterations),
                                       None if coeffs is None else ctypes.byref(coeffs), _g(g),
                                       _stream(stream)), "rodinia_hotspot_dist")
        return out_local

    def lud(self, a_local, n: int, prow: int, pcol: int, stream=None):
        """2-D block-cyclic LU (rodinia_lud_dist): this rank's local matrix (LOCAL communicator:
        the list of all ranks' local matrices), factored in place."""
        import torch
        a, keep = self._ptrs(a_local, torch.float32, "a")
        check(lib.rodinia_lud_dist(self.handle, a, int(n), int(prow), int(pcol), _stream(stream)),
              "rodinia_lud_dist")
        return a_local

    def srad(self, J_local, global_rows: int, r1, r2, c1, c2, lam: float, niter: int, g=None,
             stream=None):
        import torch
        j, keep = self._ptrs(J_local, torch.float32, "J")
        cols = (J_local[0] if self.local else J_local).shape[1]
        check(lib.rodinia_srad_dist(self.handle, j, global_rows, cols, r1, r2, c1, c2, float(lam),
                                    int(niter), _g(g), _stream(stream)), "rodinia_srad_dist")
        return J_local
