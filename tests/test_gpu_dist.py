"""Row-slab decomposition on one GPU (LOCAL communicator: all slabs on cuda:0, halos by
cudaMemcpyAsync) and the NCCL communicator at P = 1.  Sharded == single-GPU bitwise
(DESIGN.md §6), including P not dividing R and partial last exchange periods."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rg():
    import paper_conf_cgo_ivanovzdem24_b200 as m
    return m


def _split(rg, a, P):
    R = a.shape[0]
    out = []
    for r in range(P):
        r0, n = rg.dist.slab(R, P, r)
        out.append(a[r0:r0 + n].contiguous())
    return out


GRANS = [(1, 1, 1, 1, 1, 0, 0), (4, 1, 2, 1, 1, 1, 0), (4, 1, 1, 2, 4, 1, 2), (4, 1, 1, 4, 8, 1, 2 | (8 << 8)),
         (2, 1, 1, 3, 8, 1, 2)]


@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
def test_hotspot_local_slabs_bitwise(rg, P):
    R, C, iters = 203, 260, 19
    T, Pw = synth.hotspot_inputs(R, C)
    c = rg.rodinia_hotspot_coeffs_rodinia(512, 512)
    t = torch.from_numpy(T).cuda()
    p = torch.from_numpy(Pw).cuda()
    comm = rg.dist.HaloComm.local_slabs(P)
    for g in GRANS:
        ref = rg.rodinia_hotspot(t, p, iters, coeffs=c, g=g)
        ts, ps = _split(rg, t, P), _split(rg, p, P)
        outs = [torch.empty_like(x) for x in ts]
        comm.hotspot(ts, ps, outs, R, iters, coeffs=c, g=g)
        torch.cuda.synchronize()
        assert torch.equal(torch.cat(outs), ref), (P, g)
    comm.close()


def test_hotspot_slab_smaller_than_halo_rejected(rg):
    T, Pw = synth.hotspot_inputs(40, 64)
    t, p = torch.from_numpy(T).cuda(), torch.from_numpy(Pw).cuda()
    comm = rg.dist.HaloComm.local_slabs(8)  # 5 rows per slab < halo 8
    ts, ps = _split(rg, t, 8), _split(rg, p, 8)
    with pytest.raises(rg.RodiniaError) as e:
        comm.hotspot(ts, ps, [torch.empty_like(x) for x in ts], 40, 10, g=(4, 1, 1, 1, 8, 1, 2))
    assert e.value.status == rg.RODINIA_E_ILLEGAL_FACTOR


@pytest.mark.parametrize("P", [1, 2, 4, 7])
def test_srad_local_slabs_bitwise(rg, P):
    R, C, n = 150, 97, 12
    J = synth.srad_input(R, C)
    for roi in [(0, 30, 0, 40), (60, 90, 20, 50)]:
        for g in [(1, 1, 1, 1, 1, 0, 0), (2, 2, 2, 1, 1, 1, 0)]:
            ref = torch.from_numpy(J).cuda()
            rg.rodinia_srad(ref, *roi, 0.5, n, g=g)
            js = _split(rg, torch.from_numpy(J).cuda(), P)
            comm = rg.dist.HaloComm.local_slabs(P)
            comm.srad(js, R, *roi, 0.5, n, g=g)
            torch.cuda.synchronize()
            assert torch.equal(torch.cat(js), ref), (P, roi, g)
            comm.close()


def test_srad_dist_matches_oracle(rg):
    J = synth.srad_input(120, 80)
    js = _split(rg, torch.from_numpy(J).cuda(), 3)
    comm = rg.dist.HaloComm.local_slabs(3)
    comm.srad(js, 120, 10, 50, 5, 40, 0.5, 6, g=(2, 1, 1, 1, 1, 1, 0))
    got = torch.cat(js).cpu().numpy()
    ref = oracle.srad(J, 10, 50, 5, 40, 0.5, 6)
    assert np.max(np.abs(got - ref) / np.abs(ref)) <= 1e-5


def test_nccl_single_rank(rg):
    # the NCCL communicator at P = 1 (bootstrap + NCCL code path, no peers)
    import ctypes
    uid = rg.dist.unique_id()
    h = ctypes.c_void_p()
    rg.check(rg.lib.rodinia_comm_init(ctypes.byref(h), 1, 0, uid), "init")
    comm = rg.dist.HaloComm(h, 1, 0, local=False)
    T, Pw = synth.hotspot_inputs(64, 128)
    t, p = torch.from_numpy(T).cuda(), torch.from_numpy(Pw).cuda()
    out = torch.empty_like(t)
    g = (4, 1, 1, 2, 4, 1, 2)
    comm.hotspot(t, p, out, 64, 9, g=g)
    assert torch.equal(out, rg.rodinia_hotspot(t, p, 9, g=g))
    J = torch.from_numpy(synth.srad_input(64, 64)).cuda()
    J2 = J.clone()
    comm.srad(J, 64, 0, 20, 0, 20, 0.5, 5)
    rg.rodinia_srad(J2, 0, 20, 0, 20, 0.5, 5)
    assert torch.equal(J, J2)
    comm.close()


@pytest.mark.parametrize("P", [2, 3, 5, 8])
def test_srad_local_slabs_temporal_depth(rg, P):
    # halo D above / 2D below exchanged every D iterations; C % 4 == 0 while the
    # ROI-cone window is 77 or 73 columns wide at a column offset that is not a multiple of 4
    # (the window's fp64 ROI reduction must match the full grid's bit for bit)
    R, C, n = 203, 96, 12
    J = synth.srad_input(R, C)
    comm = rg.dist.HaloComm.local_slabs(P)
    for roi in [(100, 140, 5, 50), (0, 20, 30, 45)]:
        for kern in [(4, 1, 1, 2), (1, 1, 2, 1)]:
            for D in (1, 2, 4, 8):
                g = (kern[0], kern[1], kern[2], kern[3], D, 1, rg.RODINIA_STREAM if kern[0] == 4 else 0)
                g1 = g[:4] + (1,) + g[5:]
                ref = torch.from_numpy(J).cuda()
                rg.rodinia_srad(ref, *roi, 0.5, n, g=g1)
                js = _split(rg, torch.from_numpy(J).cuda(), P)
                comm.srad(js, R, *roi, 0.5, n, g=g)
                torch.cuda.synchronize()
                assert torch.equal(torch.cat(js), ref), (P, roi, g)
    comm.close()


def test_dist_buffers_reused_across_calls_and_streams(rg):
    # the communicator keeps its slab buffers; calls of different shapes and on different
    # streams stay bitwise equal to the single-GPU call (each call is ordered after the last)
    comm = rg.dist.HaloComm.local_slabs(4)
    c = rg.rodinia_hotspot_coeffs_rodinia(512, 512)
    g = (4, 1, 1, 2, 8, 1, 2)
    for (R, C, it) in [(300, 256, 17), (300, 256, 16), (190, 384, 9), (300, 256, 24)]:
        T, Pw = synth.hotspot_inputs(R, C, seed_t=R, seed_p=C)
        t, p = torch.from_numpy(T).cuda(), torch.from_numpy(Pw).cuda()
        ref = rg.rodinia_hotspot(t, p, it, coeffs=c, g=g)
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            ts, ps = _split(rg, t, 4), _split(rg, p, 4)
            outs = [torch.empty_like(x) for x in ts]
            comm.hotspot(ts, ps, outs, R, it, coeffs=c, g=g, stream=s)
        torch.cuda.synchronize()
        assert torch.equal(torch.cat(outs), ref), (R, C, it)
    comm.close()


def test_dist_schedule_matches_layout(rg):
    # the host-side schedule the library follows (rodinia_dist_schedule)
    pl = rg.dist.schedule("hotspot", 16384, 16384, 8, 3, 1000, g=(4, 1, 1, 8, 8, 1, 2 | (10 << 8)))
    assert (pl["top"], pl["bot"], pl["period"], pl["send_up"], pl["send_down"], pl["exchanges"], pl["overlap"]) == \
        (8, 8, 8, 8, 8, 125, 1)
    pl = rg.dist.schedule("srad", 8192, 8192, 8, 0, 100, roi=(0, 127, 0, 127))
    assert (pl["top"], pl["bot"], pl["period"], pl["send_up"], pl["send_down"]) == (0, 16, 8, 0, 8)
    assert (pl["cone_r0"], pl["cone_r1"], pl["cone_c0"], pl["cone_c1"]) == (0, 330, 0, 330)


def test_full_size_local_slabs_bitwise(rg):
    # BASELINE configs[2] / [3] at full size through the row-slab path with P = 8 slabs on one GPU
    # (LOCAL communicator: the same schedule, overlap split and halos as the NCCL path), in the
    # granularity the bench tunes: bitwise equal to the single-GPU solve.
    N, it = 16384, 1000
    T, Pw = synth.hotspot_inputs(N, N)
    c = rg.rodinia_hotspot_coeffs_rodinia(N, N, N * 31.25e-6, N * 31.25e-6)
    g, _ = rg.rodinia_tune_pruned("hotspot", N // 8, N, it, keep=4, reps=1)
    t, p = torch.from_numpy(T).cuda(), torch.from_numpy(Pw).cuda()
    del T, Pw
    ref = rg.rodinia_hotspot(t, p, it, coeffs=c, g=g)
    comm = rg.dist.HaloComm.local_slabs(8)
    ts, ps = _split(rg, t, 8), _split(rg, p, 8)
    outs = [torch.empty_like(x) for x in ts]
    comm.hotspot(ts, ps, outs, N, it, coeffs=c, g=g)
    torch.cuda.synchronize()
    assert torch.equal(torch.cat(outs), ref), g.astuple()
    del ts, ps, outs, ref, t, p
    M, n = 8192, 100
    J = synth.srad_input(M, M)
    for g in [(4, 1, 1, 3, 8, 1, rg.RODINIA_STREAM), None]:
        ref = torch.from_numpy(J).cuda()
        g1 = None if g is None else g[:4] + (1,) + g[5:]
        rg.rodinia_srad(ref, 0, 127, 0, 127, 0.5, n, g=g1 if g is not None else (4, 1, 1, 2, 1, 1, rg.RODINIA_STREAM))
        js = _split(rg, torch.from_numpy(J).cuda(), 8)
        comm.srad(js, M, 0, 127, 0, 127, 0.5, n, g=g)
        torch.cuda.synchronize()
        assert torch.equal(torch.cat(js), ref), g
    comm.close()
