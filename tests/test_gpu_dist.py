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
