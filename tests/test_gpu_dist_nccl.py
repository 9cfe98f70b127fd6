"""Multi-rank NCCL run of the row-slab layer: one process per visible GPU (P in {2, 4, 8} up
to the device count), torch.distributed (NCCL) only for the bootstrap and the result gather,
halos through the library's own ncclSend/ncclRecv (csrc/dist.cu).  Sharded == single-GPU bit
for bit, with R not divisible by P; the 2-D block-cyclic LU
(rodinia_lud_dist, §8(f) #3) on a prow x pcol grid equals the single-rank bits.  Skipped with fewer than two GPUs
(the builder's boxes have one; the driver's 8-GPU tier runs it)."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, ws, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=ws, device_id=torch.device("cuda", rank))
    try:
        import paper_conf_cgo_ivanovzdem24_b200 as rg
        import synth
        comm = rg.dist.HaloComm.from_process_group()
        R, C, it = 1021, 640, 37  # R % P != 0, it % D != 0
        T, P = synth.hotspot_inputs(R, C)
        c = rg.rodinia_hotspot_coeffs_rodinia(512, 512)
        r0, n = rg.rodinia_slab(R, ws, rank)
        ok = True
        for g in [(4, 1, 1, 2, 8, 1, rg.RODINIA_STREAM), (1, 1, 1, 1, 1, 0, 0), (4, 1, 1, 4, 4, 1, rg.RODINIA_STREAM)]:
            t = torch.from_numpy(T[r0:r0 + n].copy()).cuda()
            p = torch.from_numpy(P[r0:r0 + n].copy()).cuda()
            out = torch.empty_like(t)
            comm.hotspot(t, p, out, R, it, coeffs=c, g=g)
            parts = [torch.empty((rg.rodinia_slab(R, ws, r)[1], C), device="cuda") for r in range(ws)]
            dist.all_gather(parts, out)
            if rank == 0:
                ref = rg.rodinia_hotspot(torch.from_numpy(T).cuda(), torch.from_numpy(P).cuda(), it, coeffs=c, g=g)
                ok = ok and bool(torch.equal(torch.cat(parts), ref))
        J = synth.srad_input(R, C)
        for g in [(4, 1, 1, 2, 8, 1, rg.RODINIA_STREAM), (4, 1, 1, 2, 1, 1, rg.RODINIA_STREAM)]:
            js = torch.from_numpy(J[r0:r0 + n].copy()).cuda()
            comm.srad(js, R, 400, 527, 3, 130, 0.5, 20, g=g)
            parts = [torch.empty((rg.rodinia_slab(R, ws, r)[1], C), device="cuda") for r in range(ws)]
            dist.all_gather(parts, js)
            if rank == 0:
                ref = torch.from_numpy(J).cuda()
                rg.rodinia_srad(ref, 400, 527, 3, 130, 0.5, 20, g=g[:4] + (1,) + g[5:])
                ok = ok and bool(torch.equal(torch.cat(parts), ref))
        # 2-D block-cyclic LU (rodinia_lud_dist): every grid gives the single-rank bits
        nlu = 1100
        prow = 1 if ws == 2 else 2
        pcol = ws // prow
        A = torch.from_numpy(synth.lud_rodinia_matrix(nlu)).cuda()
        mine = rg.dist.block_cyclic_scatter(A, prow, pcol)[rank]
        comm.lud(mine, nlu, prow, pcol)
        gathered = [None] * ws
        dist.all_gather_object(gathered, mine.cpu())
        if rank == 0:
            got = rg.dist.block_cyclic_gather([g.cuda() for g in gathered], nlu, prow, pcol)
            one = rg.dist.HaloComm.local_slabs(1)
            ref = A.clone()
            one.lud([ref], nlu, 1, 1)
            one.close()
            ok = ok and bool(torch.equal(got, ref))
        torch.cuda.synchronize()
        comm.close()
        q.put((rank, "ok" if ok else "mismatch"))
    except Exception:  # noqa: BLE001
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("P", [2, 4, 8])
def test_nccl_multi_rank_bitwise(P):
    if not torch.cuda.is_available() or torch.cuda.device_count() < P:
        pytest.skip(f"needs {P} GPUs (have {torch.cuda.device_count() if torch.cuda.is_available() else 0})")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, P, port, q)) for r in range(P)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    for rank, msg in res:
        assert msg == "ok", f"rank {rank}:\n{msg}"
