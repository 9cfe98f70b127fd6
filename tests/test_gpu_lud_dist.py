"""GPU tests of the 2-D block-cyclic multi-GPU LU (rodinia_lud_dist) through
the LOCAL communicator (all ranks' local matrices on one device, panels moved with copies):
the same parity criteria as the single-GPU lud (reading L3: backward error, bit-exact integer
factors, forward error vs the fp64 oracle on diagonally dominant matrices), and the same bits on
every process grid (the per-element arithmetic does not depend on the distribution).
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

GRIDS = [(1, 1), (1, 2), (2, 1), (2, 2), (2, 3), (3, 2), (4, 2)]


@pytest.fixture(scope="module")
def rg():
    import paper_conf_cgo_ivanovzdem24_b200 as m
    return m


def _lu_dist(rg, A, prow, pcol):
    from paper_conf_cgo_ivanovzdem24_b200 import dist
    n = A.shape[0]
    At = torch.from_numpy(np.ascontiguousarray(A, np.float32)).cuda()
    parts = dist.block_cyclic_scatter(At, prow, pcol)
    for r, x in enumerate(parts):
        assert tuple(x.shape) == dist.lud_layout(n, prow, pcol, r)
    comm = dist.HaloComm.local_slabs(prow * pcol)
    try:
        comm.lud(parts, n, prow, pcol)
        torch.cuda.synchronize()
    finally:
        comm.close()
    return dist.block_cyclic_gather(parts, n, prow, pcol)


def _backward(A, p):
    p = p.double()
    n = p.shape[0]
    L = torch.tril(p, -1) + torch.eye(n, dtype=p.dtype, device=p.device)
    U = torch.triu(p)
    Ad = torch.from_numpy(np.asarray(A, np.float64)).to(p.device)
    return float((Ad - L @ U).abs().max() / Ad.abs().max())


@pytest.mark.parametrize("n", [1, 100, 128, 129, 300, 1000, 1100])
def test_backward_error_and_grid_independence(rg, n):
    A = synth.lud_rodinia_matrix(n)
    ref = _lu_dist(rg, A, 1, 1)
    assert _backward(A, ref) <= 1e-5, n
    for prow, pcol in GRIDS[1:]:
        got = _lu_dist(rg, A, prow, pcol)
        assert torch.equal(got, ref), (n, prow, pcol)


@pytest.mark.parametrize("n", [7, 300, 777])
def test_integer_factors_bit_exact(rg, n):
    A, L0, U0 = synth.lud_integer_factors(n)
    for prow, pcol in [(1, 1), (2, 2), (3, 2)]:
        L, U = oracle.lud_unpack(_lu_dist(rg, A, prow, pcol).cpu().numpy())
        assert np.array_equal(L, L0) and np.array_equal(U, U0), (n, prow, pcol)


@pytest.mark.parametrize("n", [300, 1024])
def test_forward_error_diag_dominant(rg, n):
    A = synth.lud_diag_dominant(n)
    L64, U64 = oracle.lud_unpack(oracle.lud(A))
    L, U = oracle.lud_unpack(_lu_dist(rg, A, 2, 2).cpu().numpy().astype(np.float64))
    assert np.abs(L - L64).max() / np.abs(L64).max() <= 1e-5
    assert np.abs(U - U64).max() / np.abs(U64).max() <= 1e-5


def test_full_size_backward_error_2x4(rg):
    # BASELINE configs[4] size (8192) on a 2 x 4 grid: backward error on a row sample
    n = 8192
    A = synth.lud_rodinia_matrix(n)
    p = _lu_dist(rg, A, 2, 4).double()
    L = torch.tril(p, -1) + torch.eye(n, dtype=p.dtype, device=p.device)
    U = torch.triu(p)
    rows = torch.arange(0, n, 61, device=p.device)
    Ad = torch.from_numpy(A[rows.cpu().numpy()].astype(np.float64)).to(p.device)
    assert float((Ad - L[rows] @ U).abs().max() / abs(A).max()) <= 1e-5


def test_bad_grid(rg):
    from paper_conf_cgo_ivanovzdem24_b200 import dist
    comm = dist.HaloComm.local_slabs(4)
    try:
        A = torch.zeros((256, 256), device="cuda")
        parts = dist.block_cyclic_scatter(A, 2, 2)
        with pytest.raises(rg.RodiniaError):
            comm.lud(parts, 256, 1, 3)
    finally:
        comm.close()
