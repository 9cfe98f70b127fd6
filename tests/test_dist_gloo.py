"""World-size-2 CPU tests (gloo) of the multi-GPU row-slab layer's host logic.

(a) bootstrap: rank 0 creates the NCCL unique id through the library, torch.distributed ships
    it, both ranks hold the same 128 bytes (what rodinia_comm_init consumes);
(b) the decomposition protocol of csrc/dist.cu -- slab partition (rodinia_slab), halo depths
    (hotspot D/D, srad D above / 2D below), exchange schedule (first rows up, last rows down,
    every D steps), clamping at buffer edges, srad q0sqr(t) from the ROI dependency cone --
    replayed with the CPU oracle as the per-slab solver and gloo send/recv as the transport:
    the gathered result must equal the single-grid oracle bit for bit.
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _exchange(buf, top, own, bot, up, down, rank, ws):
    """Send my first `up` own rows up / last `down` own rows down; receive the halos."""
    reqs = []
    if rank > 0:
        reqs.append(dist.isend(torch.from_numpy(buf[top:top + up].copy()), rank - 1))
        recv_top = torch.empty((down, buf.shape[1]), dtype=torch.float64)
        reqs.append(dist.irecv(recv_top, rank - 1))
    if rank + 1 < ws:
        reqs.append(dist.isend(torch.from_numpy(buf[top + own - down:top + own].copy()), rank + 1))
        recv_bot = torch.empty((up, buf.shape[1]), dtype=torch.float64)
        reqs.append(dist.irecv(recv_bot, rank + 1))
    for r in reqs:
        r.wait()
    if rank > 0:
        buf[:down] = recv_top.numpy()
    if rank + 1 < ws:
        buf[top + own:top + own + up] = recv_bot.numpy()


def _gather_rows(x, ws):
    parts = [None] * ws
    dist.all_gather_object(parts, x)
    return np.concatenate(parts, axis=0)


def _worker(rank, ws, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        import oracle
        import paper_conf_cgo_ivanovzdem24_b200 as rg
        import synth

        # (a) bootstrap of the NCCL unique id over the process group
        obj = [rg.dist.unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        ids = [None] * ws
        dist.all_gather_object(ids, obj[0])
        assert len(ids[0]) == 128 and all(i == ids[0] for i in ids)

        # (b1) hotspot: halo D = steps per exchange, iterations not a multiple of D
        R, C, iters, D = 37, 23, 11, 3
        T, P = synth.hotspot_inputs(R, C)
        cf = oracle.hotspot_coeffs_rodinia(512, 512)
        r0, own = rg.dist.slab(R, ws, rank)
        top = D if rank > 0 else 0
        bot = D if rank + 1 < ws else 0
        buf = np.zeros((top + own + bot, C))
        pw = np.zeros_like(buf)
        buf[top:top + own] = T[r0:r0 + own]
        pw[top:top + own] = P[r0:r0 + own]
        _exchange(pw, top, own, bot, D, D, rank, ws)
        done = 0
        while done < iters:
            steps = min(D, iters - done)
            _exchange(buf, top, own, bot, D, D, rank, ws)
            buf = oracle.hotspot(buf, pw, steps, **cf)   # clamps at the buffer edges
            done += steps
        full = _gather_rows(buf[top:top + own], ws)
        assert np.array_equal(full, oracle.hotspot(T, P, iters, **cf))

        # (b2) srad: halo D above, 2D below; q0sqr(t) from the ROI cone window
        R, C, n, D, lam = 41, 30, 7, 1, 0.5
        r1, r2, c1, c2 = 25, 33, 4, 12           # ROI owned by rank 1, read by both
        J = synth.srad_input(R, C)
        w = J[max(0, r1 - n):min(R, r2 + 2 * n + 3), max(0, c1 - n):min(C, c2 + 2 * n + 3)]
        _, q0 = oracle.srad(w, r1 - max(0, r1 - n), r2 - max(0, r1 - n), c1 - max(0, c1 - n),
                            c2 - max(0, c1 - n), lam, n, return_q0=True)
        _, q0_full = oracle.srad(J, r1, r2, c1, c2, lam, n, return_q0=True)
        assert np.array_equal(q0, q0_full)       # the cone reproduces q0sqr(t) exactly
        r0, own = rg.dist.slab(R, ws, rank)
        top = D if rank > 0 else 0
        bot = 2 * D if rank + 1 < ws else 0
        buf = np.zeros((top + own + bot, C))
        buf[top:top + own] = J[r0:r0 + own]
        for t in range(0, n, D):
            _exchange(buf, top, own, bot, 2 * D, D, rank, ws)
            for k in range(t, min(n, t + D)):
                buf = oracle.srad_step(buf, q0[k], lam)
        full = _gather_rows(buf[top:top + own], ws)
        assert np.array_equal(full, oracle.srad(J, r1, r2, c1, c2, lam, n))

        # negative control: srad with only D rows below is NOT equal (the 2-row reach)
        top, bot = (D if rank > 0 else 0), (D if rank + 1 < ws else 0)
        buf = np.zeros((top + own + bot, C))
        buf[top:top + own] = J[r0:r0 + own]
        for t in range(n):
            _exchange(buf, top, own, bot, D, D, rank, ws)
            buf = oracle.srad_step(buf, q0[t], lam)
        bad = _gather_rows(buf[top:top + own], ws)
        assert not np.array_equal(bad, oracle.srad(J, r1, r2, c1, c2, lam, n))
        q.put((rank, "ok"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


def test_slab_protocol_world_size_2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, msg in res:
        assert msg == "ok", f"rank {rank}:\n{msg}"


def test_slab_partition():
    import paper_conf_cgo_ivanovzdem24_b200 as rg
    for R, P in [(16384, 8), (61, 8), (10, 3), (7, 7)]:
        rows = [rg.dist.slab(R, P, r) for r in range(P)]
        assert rows[0][0] == 0 and sum(n for _, n in rows) == R
        for (a, n), (b, _) in zip(rows, rows[1:]):
            assert a + n == b
        assert max(n for _, n in rows) - min(n for _, n in rows) <= 1
