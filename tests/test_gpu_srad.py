"""GPU parity of srad_v2 against the fp64 oracle (through the C ABI).

Tolerance 1e-5 relative elementwise (north_star; J stays in [1, e)).  Every variant is bitwise
identical to the Rodinia-dataflow (uncoarsened) variant.
"""
import numpy as np
import pytest

import oracle
import synth
from tests._util import rel_err, srad_window_block

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = 1e-5
UNC = (1, 1, 1, 1, 1, 0, 0)


@pytest.fixture(scope="module")
def rg():
    import paper_conf_cgo_ivanovzdem24_b200 as m
    return m


def _run(rg, J, roi, lam, n, g):
    t = torch.from_numpy(np.ascontiguousarray(J, np.float32)).cuda()
    rg.rodinia_srad(t, *roi, lam, n, g=g)
    rg.rodinia_sync()
    return t.cpu().numpy()


def _roi(R, C):
    return (0, min(127, R - 1), 0, min(127, C - 1))


@pytest.mark.parametrize("R,C", [(1, 1), (1, 40), (33, 1), (16, 16), (37, 53), (100, 131), (257, 515)])
def test_vs_oracle(rg, R, C):
    J = synth.srad_input(R, C)
    roi = _roi(R, C)
    for n in (1, 5, 20):
        ref = oracle.srad(J, *roi, 0.5, n)
        for g in (UNC, (4, 1, 2, 2, 1, 1, 0), (4, 1, 1, 2, 1, 1, 2)):
            got = _run(rg, J, roi, 0.5, n, g)
            assert rel_err(got, ref) <= TOL, (R, C, n, g, rel_err(got, ref))


def test_interior_roi_and_lambda(rg):
    J = synth.srad_input(90, 70, seed=11)
    roi = (20, 50, 10, 40)
    for lam in (0.1, 0.5, 1.0):
        ref = oracle.srad(J, *roi, lam, 8)
        assert rel_err(_run(rg, J, roi, lam, 8, (2, 2, 1, 1, 1, 1, 0)), ref) <= TOL


def _fused_grans():
    out = []
    for tx, ty in [(1, 1), (1, 2), (2, 1), (2, 2), (1, 4), (4, 1), (4, 2), (2, 4), (4, 4), (8, 1), (1, 8), (8, 2)]:
        for mode in (0, 1):
            for bx, by in [(1, 1), (3, 2), (2, 5)]:
                if (tx, ty, mode, bx, by) == (1, 1, 0, 1, 1):
                    continue
                out.append((tx, ty, bx, by, 1, mode, 0))
    return out


def _stream_grans(rg):
    out = []
    for r in rg.rodinia_variants("srad"):
        g = r["g"]
        if (g[6] & rg.RODINIA_STREAM) and r["status"] == 0:
            for bx, by in [(1, 1), (2, 3), (1, 8)]:
                out.append((g[0], 1, bx, by, 1, 1, g[6]))
    assert out
    return out


@pytest.mark.parametrize("R,C,niter", [(131, 97, 6), (70, 256, 6), (33, 260, 6), (300, 516, 7), (181, 260, 5)])
def test_all_variants_bit_identical(rg, R, C, niter):
    # 300 x 516 has interior chunks/bands (the stream family's fast path) next to edge ones
    J = synth.srad_input(R, C, seed=3)
    roi = (0, min(60, R - 1), 5, 70)
    base = _run(rg, J, roi, 0.5, niter, UNC)
    assert rel_err(base, oracle.srad(J, *roi, 0.5, niter)) <= TOL
    for g in _fused_grans() + _stream_grans(rg):
        assert np.array_equal(_run(rg, J, roi, 0.5, niter, g), base), g


def test_uniform_and_lambda_zero_unchanged(rg):
    J = np.full((64, 96), 2.0, np.float32)
    for g in (UNC, (4, 1, 2, 2, 1, 1, 0)):
        assert np.array_equal(_run(rg, J, (0, 31, 0, 31), 0.5, 25, g), J)
    J = synth.srad_input(50, 60)
    assert np.array_equal(_run(rg, J, (0, 20, 0, 20), 0.0, 5, (2, 2, 1, 1, 1, 0, 0)), J)


@pytest.mark.parametrize("g", [UNC, (4, 1, 1, 1, 1, 1, 2)])
def test_degenerate_roi_reported(rg, g):
    J = synth.srad_input(40, 40)
    J[:4, :4] = 0.0
    t = torch.from_numpy(J).cuda()
    rg.rodinia_srad(t, 0, 3, 0, 3, 0.5, 3, g=g)  # asynchronous: returns before the check
    with pytest.raises(rg.RodiniaError) as e:
        rg.rodinia_sync()
    assert e.value.status == rg.RODINIA_E_DEGENERATE
    assert np.array_equal(t.cpu().numpy(), J)  # J left as of the failing (first) iteration
    rg.rodinia_sync()  # sticky status cleared


def test_full_size_windows(rg):
    # BASELINE configs[3]: 8192^2, 100 iterations, ROI (0,127,0,127), lambda 0.5, in the launch
    # configuration bench.py times (the TDO winner of its rodinia_tune call).  Three 64 x 64
    # output windows -- the corner holding the ROI, a right-edge strip and the interior -- are
    # compared elementwise with the windowed oracle driven by the exact q0sqr sequence (taken
    # from the ROI's dependency cone, rows/cols [0, 127 + 2*100 + margin], reading S10).
    N, n, lam = 8192, 100, 0.5
    J = synth.srad_input(N, N)
    w = 127 + 2 * n + 8
    _, q0 = oracle.srad(J[:w, :w], 0, 127, 0, 127, lam, n, return_q0=True)
    g, _ = rg.rodinia_tune("srad", N, N, n, reps=2)
    t = torch.from_numpy(J).cuda()
    rg.rodinia_srad(t, 0, 127, 0, 127, lam, n, g=g)
    out = t.cpu().numpy()
    assert np.isfinite(out).all()
    for (i0, j0) in [(0, 0), (3000, N - 64), (4000, 5000)]:
        ref = srad_window_block(J, i0, j0, 64, 64, n, q0, lam)
        got = out[i0:i0 + 64, j0:j0 + 64]
        assert rel_err(got, ref) <= TOL, (g.astuple(), i0, j0, rel_err(got, ref))
    # whole-grid cross-variant equality at full size (10 iterations)
    a = torch.from_numpy(J).cuda()
    b = torch.from_numpy(J).cuda()
    rg.rodinia_srad(a, 0, 127, 0, 127, lam, 10, g=g)
    rg.rodinia_srad(b, 0, 127, 0, 127, lam, 10, g=UNC)
    assert torch.equal(a, b)


def test_host_entry(rg):
    J = synth.srad_input(70, 90)
    got = rg.rodinia_srad_host(J, 0, 30, 0, 30, 0.5, 4, g=(2, 1, 1, 1, 1, 1, 0))
    assert rel_err(got, oracle.srad(J, 0, 30, 0, 30, 0.5, 4)) <= TOL
