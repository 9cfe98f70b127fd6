"""CPU tests (gloo, world sizes 2 and 4) of the 2-D block-cyclic LU's host logic
(rodinia_lud_dist, csrc/dist.cu):

(a) the local layout the library reports (rodinia_lud_dist_layout) is the block-cyclic one:
    block (I, J) of 128 x 128 on rank (I mod prow, J mod pcol), local blocks in increasing order;
(b) the protocol dist.cu runs -- per block column k the owner of A_kk factors it and broadcasts
    it, process column k mod pcol solves L_Ik = A_Ik U_kk^-1, process row k mod prow solves
    U_kJ = L_kk^-1 A_kJ, L panels travel along process rows and U panels along process columns
    (send/recv), every rank updates its trailing blocks -- executed with gloo as the transport
    and fp64 arithmetic (the oracle's Doolittle for the diagonal block, scipy's triangular
    solves for the panels), reproduces the fp64 oracle's LU of the whole matrix.
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402

NB = 128


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _idx(n, P, p):
    nb = (n + NB - 1) // NB
    parts = [np.arange(I * NB, min(n, (I + 1) * NB)) for I in range(p, nb, P)]
    return np.concatenate(parts) if parts else np.zeros(0, dtype=np.int64)


def _blocks_le(k, P, p):
    return 0 if k < p else (k - p) // P + 1


def _worker(rank, ws, prow, pcol, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        from scipy.linalg import solve_triangular

        import oracle
        import paper_conf_cgo_ivanovzdem24_b200 as rg
        import synth

        for n in (300, 517):
            A = synth.lud_rodinia_matrix(n).astype(np.float64)
            pr, pc = rank // pcol, rank % pcol
            ri, ci = _idx(n, prow, pr), _idx(n, pcol, pc)
            assert (len(ri), len(ci)) == rg.dist.lud_layout(n, prow, pcol, rank)
            loc = A[np.ix_(ri, ci)].copy()
            nb = (n + NB - 1) // NB
            for k in range(nb):
                pk, qk = k % prow, k % pcol
                root = pk * pcol + qk
                bk = min(NB, n - k * NB)
                lrk, lck = (k // prow) * NB, (k // pcol) * NB
                dk = torch.zeros((bk, bk), dtype=torch.float64)
                if rank == root:
                    dk = torch.from_numpy(oracle.lud(loc[lrk:lrk + bk, lck:lck + bk]))
                    loc[lrk:lrk + bk, lck:lck + bk] = dk.numpy()
                if k == nb - 1:
                    break
                dist.broadcast(dk, src=root)
                Lkk = np.tril(dk.numpy(), -1) + np.eye(bk)
                Ukk = np.triu(dk.numpy())
                lr0, lc0 = _blocks_le(k, prow, pr) * NB, _blocks_le(k, pcol, pc) * NB
                rows, cols = loc.shape[0] - lr0, loc.shape[1] - lc0
                if pc == qk and rows > 0:   # L_Ik = A_Ik U_kk^-1
                    loc[lr0:, lck:lck + NB] = solve_triangular(Ukk, loc[lr0:, lck:lck + NB].T, trans="T",
                                                               lower=False).T
                if pr == pk and cols > 0:   # U_kJ = L_kk^-1 A_kJ
                    loc[lrk:lrk + NB, lc0:] = solve_triangular(Lkk, loc[lrk:lrk + NB, lc0:], lower=True,
                                                               unit_diagonal=True)
                # panels: L along process rows from (pr, qk), U along process columns from (pk, pc)
                Lp = torch.from_numpy(np.ascontiguousarray(loc[lr0:, lck:lck + NB])) if pc == qk else \
                    torch.empty((rows, NB), dtype=torch.float64)
                Up = torch.from_numpy(np.ascontiguousarray(loc[lrk:lrk + NB, lc0:])) if pr == pk else \
                    torch.empty((NB, cols), dtype=torch.float64)
                reqs = []
                if rows > 0 and pcol > 1:
                    if pc == qk:
                        reqs += [dist.isend(Lp, pr * pcol + c) for c in range(pcol) if c != qk]
                    else:
                        reqs.append(dist.irecv(Lp, pr * pcol + qk))
                if cols > 0 and prow > 1:
                    if pr == pk:
                        reqs += [dist.isend(Up, p * pcol + pc) for p in range(prow) if p != pk]
                    else:
                        reqs.append(dist.irecv(Up, pk * pcol + pc))
                for r in reqs:
                    r.wait()
                if rows > 0 and cols > 0:
                    loc[lr0:, lc0:] -= Lp.numpy() @ Up.numpy()
            parts = [None] * ws
            dist.all_gather_object(parts, loc)
            full = np.empty((n, n))
            for r, x in enumerate(parts):
                full[np.ix_(_idx(n, prow, r // pcol), _idx(n, pcol, r % pcol))] = x
            ref = oracle.lud(A)
            assert np.abs(full - ref).max() <= 1e-9 * np.abs(ref).max(), n
        q.put((rank, "ok"))
    except Exception:  # noqa: BLE001
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("prow,pcol", [(1, 2), (2, 1), (2, 2)])
def test_block_cyclic_protocol(prow, pcol):
    ws = prow * pcol
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, ws, prow, pcol, port, q)) for r in range(ws)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, msg in res:
        assert msg == "ok", f"rank {rank}:\n{msg}"


def test_layout_block_cyclic():
    import paper_conf_cgo_ivanovzdem24_b200 as rg
    for n, prow, pcol in [(1, 1, 1), (300, 2, 3), (1100, 4, 2), (8192, 2, 4), (100, 3, 3)]:
        m_tot = sum(rg.dist.lud_layout(n, prow, pcol, r * pcol)[0] for r in range(prow))
        n_tot = sum(rg.dist.lud_layout(n, prow, pcol, c)[1] for c in range(pcol))
        assert m_tot == n and n_tot == n
        for r in range(prow * pcol):
            assert rg.dist.lud_layout(n, prow, pcol, r) == (len(_idx(n, prow, r // pcol)), len(_idx(n, pcol, r % pcol)))
    with pytest.raises(rg.RodiniaError):
        rg.dist.lud_layout(100, 2, 2, 4)


def test_lud_dist_argument_validation_without_device():
    # rodinia_lud_dist refuses a process grid that does not match the communicator, null local
    # matrices and bad sizes before any CUDA call (no device needed)
    import ctypes

    import paper_conf_cgo_ivanovzdem24_b200 as rg
    h = ctypes.c_void_p()
    assert rg.lib.rodinia_comm_init_local(ctypes.byref(h), 4) == rg.RODINIA_OK
    try:
        arr = (ctypes.c_void_p * 4)(1, 1, 1, 1)
        a = ctypes.cast(arr, ctypes.c_void_p)
        assert rg.lib.rodinia_lud_dist(h, a, 256, 1, 3, None) == rg.RODINIA_E_INVALID  # 1 x 3 != 4
        assert rg.lib.rodinia_lud_dist(h, a, 0, 2, 2, None) == rg.RODINIA_E_INVALID
        assert rg.lib.rodinia_lud_dist(h, None, 256, 2, 2, None) == rg.RODINIA_E_INVALID
        assert rg.lib.rodinia_lud_dist(None, a, 256, 2, 2, None) == rg.RODINIA_E_INVALID
    finally:
        rg.lib.rodinia_comm_destroy(h)
