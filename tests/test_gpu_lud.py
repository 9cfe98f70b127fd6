"""GPU parity of blocked lud (reading L3 of DESIGN.md):
 (i) backward error max|A - L U| / max|A| <= 1e-5 (product in fp64) on Rodinia's matrix;
 (ii) per-factor normwise forward error vs the fp64 oracle <= 1e-5 on diagonally dominant
      random matrices;
 (iii) bit-exact recovery of integer factors (every fp32 operation exact);
 plus bitwise equality of all (t, b) variants for a fixed panel width.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

UNC = (1, 1, 1, 1, 1, 0, 0)


@pytest.fixture(scope="module")
def rg():
    import paper_conf_cgo_ivanovzdem24_b200 as m
    return m


def _lu(rg, A, panel=16, g=UNC):
    t = torch.from_numpy(np.ascontiguousarray(A, np.float32)).cuda()
    rg.rodinia_lud(t, panel, g=g)
    torch.cuda.synchronize()
    return t


def _unpack_t(p):
    n = p.shape[0]
    L = torch.tril(p, -1) + torch.eye(n, dtype=p.dtype, device=p.device)
    return L, torch.triu(p)


def _backward(A, packed):
    p = packed.double()
    L, U = _unpack_t(p)
    Ad = torch.from_numpy(np.asarray(A, np.float64)).to(p.device)
    return float((Ad - L @ U).abs().max() / Ad.abs().max())


@pytest.mark.parametrize("n", [1, 2, 15, 16, 17, 33, 100, 257, 1000])
@pytest.mark.parametrize("panel", [16, 32])
def test_backward_error_rodinia_matrix(rg, n, panel):
    A = synth.lud_rodinia_matrix(n)
    for g in (UNC, (2, 1, 3, 2, 1, 1, 0)):
        assert _backward(A, _lu(rg, A, panel, g)) <= 1e-5, (n, panel, g)


@pytest.mark.parametrize("n", [64, 300, 1024, 2048])
def test_forward_error_diag_dominant(rg, n):
    A = synth.lud_diag_dominant(n)
    L64, U64 = oracle.lud_unpack(oracle.lud(A))
    for panel in (16, 32):
        p = _lu(rg, A, panel, (2, 2, 4, 1, 1, 1, 0)).cpu().numpy().astype(np.float64)
        L, U = oracle.lud_unpack(p)
        assert np.abs(L - L64).max() / np.abs(L64).max() <= 1e-5
        assert np.abs(U - U64).max() / np.abs(U64).max() <= 1e-5


@pytest.mark.parametrize("n", [7, 300, 512])
def test_integer_factors_bit_exact(rg, n):
    A, L0, U0 = synth.lud_integer_factors(n)
    for panel in (16, 32):
        for g in (UNC, (4, 4, 2, 7, 1, 0, 0), (8, 1, 1, 1, 1, 1, 0)):
            try:
                p = _lu(rg, A, panel, g).cpu().numpy()
            except rg.RodiniaError as e:
                assert e.status in (rg.RODINIA_E_NOT_BUILT, rg.RODINIA_E_ILLEGAL_FACTOR)
                continue
            L, U = oracle.lud_unpack(p)
            assert np.array_equal(L, L0) and np.array_equal(U, U0), (n, panel, g)


def test_all_variants_bit_identical(rg):
    A = synth.lud_rodinia_matrix(200)
    for panel in (16, 32):
        base = _lu(rg, A, panel, UNC).cpu().numpy()
        for r in rg.rodinia_variants("lud"):
            g = r["g"]
            stream = bool(g[6] & rg.RODINIA_STREAM)
            for bx, by in ([(1, 1), (1, 5)] if stream else [(1, 1), (2, 1), (7, 3)]):
                # RODINIA_FORCE: the ptxas-pruned (spilling) instantiations must agree bitwise too
                gg = (g[0], g[1], bx, by, 1, g[5], g[6] | rg.RODINIA_FORCE)
                try:
                    got = _lu(rg, A, panel, gg).cpu().numpy()
                except rg.RodiniaError as e:
                    assert e.status in (rg.RODINIA_E_NOT_BUILT, rg.RODINIA_E_ILLEGAL_FACTOR), gg
                    continue
                assert np.array_equal(got, base), (panel, gg)


def test_triangular_and_identity(rg):
    rng = np.random.default_rng(2)
    U = (np.triu(rng.random((40, 40))) + np.eye(40)).astype(np.float32)
    p = _lu(rg, U).cpu().numpy()
    assert np.array_equal(np.triu(p), U) and np.all(np.tril(p, -1) == 0)
    I = np.eye(48, dtype=np.float32)
    assert np.array_equal(_lu(rg, I, 16, (4, 1, 2, 2, 1, 1, 0)).cpu().numpy(), I)


def test_full_size_8192_backward_error(rg):
    # BASELINE configs[4]: 8192^2 fp32, default (bench) launch configuration
    n = 8192
    A = synth.lud_rodinia_matrix(n)
    p = _lu(rg, A, 16, None)
    assert _backward(A, p) <= 1e-5
    assert torch.equal(p, _lu(rg, A, 16, UNC))  # tuned/default vs uncoarsened: bit-identical


def test_host_entry(rg):
    A = synth.lud_diag_dominant(100)
    got = rg.rodinia_lud_host(A, 16, g=(2, 1, 2, 1, 1, 1, 0))
    L, U = oracle.lud_unpack(got.astype(np.float64))
    assert np.abs(L @ U - A).max() / np.abs(A).max() <= 1e-5


# ---------------------------------------------------------------- panel 128: tensor cores
# Two-level blocking with the rank-128 trailing update on tcgen05 (kind::tf32, 3xTF32 split;
# DESIGN.md §5).  Same parity criteria (L3); integer factors stay bit-exact because every
# operand is exactly a TF32 value (lo parts are 0) and every partial sum is an exact integer.
@pytest.mark.parametrize("n", [1, 17, 100, 128, 129, 257, 300, 1000, 1100])
def test_tc_backward_error_rodinia_matrix(rg, n):
    A = synth.lud_rodinia_matrix(n)
    assert _backward(A, _lu(rg, A, 128)) <= 1e-5, n


@pytest.mark.parametrize("n", [300, 1024, 2048])
def test_tc_forward_error_diag_dominant(rg, n):
    A = synth.lud_diag_dominant(n)
    L64, U64 = oracle.lud_unpack(oracle.lud(A))
    p = _lu(rg, A, 128).cpu().numpy().astype(np.float64)
    L, U = oracle.lud_unpack(p)
    assert np.abs(L - L64).max() / np.abs(L64).max() <= 1e-5
    assert np.abs(U - U64).max() / np.abs(U64).max() <= 1e-5


@pytest.mark.parametrize("n", [7, 300, 512, 777])
def test_tc_integer_factors_bit_exact(rg, n):
    A, L0, U0 = synth.lud_integer_factors(n)
    L, U = oracle.lud_unpack(_lu(rg, A, 128).cpu().numpy())
    assert np.array_equal(L, L0) and np.array_equal(U, U0), n


def test_tc_full_size_backward_error(rg):
    # BASELINE configs[4] size (8192), Rodinia matrix; backward error via an fp64 product on
    # the GPU (1.1e12 flop) on a row sample of A - L U
    n = 8192
    A = synth.lud_rodinia_matrix(n)
    p = _lu(rg, A, 128).double()
    L, U = _unpack_t(p)
    rows = torch.arange(0, n, 61, device=p.device)
    Ad = torch.from_numpy(A[rows.cpu().numpy()].astype(np.float64)).to(p.device)
    err = float((Ad - L[rows] @ U).abs().max() / abs(A).max())
    assert err <= 1e-5, err


def test_concurrent_calls_same_n_two_streams(rg):
    # Two factorisations of the same size on two streams share one cached graph; each must
    # factor its own matrix (the slot write is the graph's root node, updated per launch).
    n = 2048
    A1 = synth.lud_rodinia_matrix(n)
    A2 = synth.lud_diag_dominant(n)
    for panel in (16, 128):
        r1 = _lu(rg, A1, panel).clone()
        r2 = _lu(rg, A2, panel).clone()
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        for _ in range(3):
            t1 = torch.from_numpy(A1).cuda()
            t2 = torch.from_numpy(A2).cuda()
            torch.cuda.synchronize()
            rg.rodinia_lud(t1, panel, g=UNC, stream=s1)
            rg.rodinia_lud(t2, panel, g=UNC, stream=s2)
            torch.cuda.synchronize()
            assert torch.equal(t1, r1) and torch.equal(t2, r2), panel


def test_unaligned_matrix_view(rg):
    # an offset view (not 16-byte aligned) is factored bit-identically to an aligned copy
    n = 300
    A = synth.lud_rodinia_matrix(n)
    for panel in (16, 32, 128):
        ref = _lu(rg, A, panel, (2, 2, 2, 2, 1, 1, 0) if panel != 128 else UNC)
        buf = torch.empty(n * n + 1, device="cuda")
        v = buf[1:].view(n, n)
        v.copy_(torch.from_numpy(A))
        rg.rodinia_lud(v, panel, g=(2, 2, 2, 2, 1, 1, 0) if panel != 128 else UNC)
        torch.cuda.synchronize()
        assert torch.equal(v, ref), panel
