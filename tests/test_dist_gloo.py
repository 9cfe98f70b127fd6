"""World-size-2 CPU tests (gloo) of the multi-GPU row-slab layer's host logic.

(a) bootstrap: rank 0 creates the NCCL unique id through the library, torch.distributed ships
    it, both ranks hold the same 128 bytes (what rodinia_comm_init consumes);
(b) the decomposition csrc/dist.cu executes, taken from the library itself: every rank asks
    rodinia_dist_schedule (host-only C ABI) for its slab, halo depths, exchange period and
    sizes, overlap split and (srad) ROI-cone window, and runs exactly that schedule with the CPU
    oracle as the per-slab solver and gloo send/recv as the transport -- including the hotspot
    overlap split (interior from the owned rows alone, boundary strips of D halo + 2D owned
    rows).  The gathered result must equal the single-grid oracle bit for bit, for several
    temporal depths D and a rank count that does not divide the rows.
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

        # (b1) hotspot: the library's schedule for D = 1, 2, 3 (iterations not a multiple of D)
        R, C, iters = 37, 23, 11
        T, P = synth.hotspot_inputs(R, C)
        cf = oracle.hotspot_coeffs_rodinia(512, 512)
        for D in (1, 2, 3):
            g = (1, 1, 1, 1, 1, 0, 0) if D == 1 else (4, 1, 1, 1, D, 1, rg.RODINIA_STREAM)
            if D == 3:
                g = (2, 1, 1, 1, 4, 1, rg.RODINIA_STREAM)  # h = 4
            pl = rg.dist.schedule("hotspot", R, C, ws, rank, iters, g=g)
            D = pl["period"]
            r0, own, top, bot = pl["row0"], pl["own"], pl["top"], pl["bot"]
            assert (r0, own) == rg.dist.slab(R, ws, rank)
            buf = np.zeros((top + own + bot, C))
            pw = np.zeros_like(buf)
            buf[top:top + own] = T[r0:r0 + own]
            pw[top:top + own] = P[r0:r0 + own]
            _exchange(pw, top, own, bot, pl["send_up"] or D, pl["send_down"] or D, rank, ws)
            done = nex = 0
            while done < iters:
                steps = min(D, iters - done)
                _exchange(buf, top, own, bot, pl["send_up"] or D, pl["send_down"] or D, rank, ws)
                nex += 1
                if pl["overlap"] and steps == D:
                    # interior: owned rows only -> rows [D, own - D) exact
                    inner = oracle.hotspot(buf[top:top + own], pw[top:top + own], steps, **cf)
                    new = np.zeros_like(buf)
                    new[top + D:top + own - D] = inner[D:own - D]
                    ts = oracle.hotspot(buf[:top + 2 * D], pw[:top + 2 * D], steps, **cf)
                    new[top:top + D] = ts[top:top + D]
                    b0 = top + own - 2 * D
                    bs = oracle.hotspot(buf[b0:], pw[b0:], steps, **cf)
                    new[top + own - D:top + own] = bs[D:2 * D]
                    buf = new
                else:
                    buf = oracle.hotspot(buf, pw, steps, **cf)   # clamps at the buffer edges
                done += steps
            assert nex == pl["exchanges"]
            full = _gather_rows(buf[top:top + own], ws)
            assert np.array_equal(full, oracle.hotspot(T, P, iters, **cf)), D

        # (b2) srad: the library's schedule (halo D above, 2D below, exchange every D iterations)
        # and its ROI-cone window for q0sqr(t)
        R, C, n, lam = 41, 30, 7, 0.5
        r1, r2, c1, c2 = 25, 33, 4, 12           # ROI owned by rank 1, read by both
        J = synth.srad_input(R, C)
        _, q0_full = oracle.srad(J, r1, r2, c1, c2, lam, n, return_q0=True)
        ref = oracle.srad(J, r1, r2, c1, c2, lam, n)
        for Dg in (1, 2, 3, 0):
            g = None if Dg == 0 else (4, 1, 1, 2, Dg, 1, rg.RODINIA_STREAM)
            pl = rg.dist.schedule("srad", R, C, ws, rank, n, roi=(r1, r2, c1, c2), g=g)
            D = pl["period"]
            assert pl["top"] in (0, D) and pl["bot"] in (0, 2 * D)
            w0, w1, v0, v1 = pl["cone_r0"], pl["cone_r1"], pl["cone_c0"], pl["cone_c1"]
            _, q0 = oracle.srad(J[w0:w1, v0:v1], r1 - w0, r2 - w0, c1 - v0, c2 - v0, lam, n, return_q0=True)
            assert np.array_equal(q0, q0_full)       # the cone reproduces q0sqr(t) exactly
            r0, own, top, bot = pl["row0"], pl["own"], pl["top"], pl["bot"]
            buf = np.zeros((top + own + bot, C))
            buf[top:top + own] = J[r0:r0 + own]
            for t in range(0, n, D):
                _exchange(buf, top, own, bot, 2 * D, D, rank, ws)
                for k in range(t, min(n, t + D)):
                    buf = oracle.srad_step(buf, q0[k], lam)
            full = _gather_rows(buf[top:top + own], ws)
            assert np.array_equal(full, ref), Dg
        D = 1
        r0, own = rg.dist.slab(R, ws, rank)
        q0 = q0_full

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
