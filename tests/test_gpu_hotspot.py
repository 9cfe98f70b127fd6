"""GPU parity of the hotspot kernels against the fp64 oracle (through the C ABI).

Tolerance: 1e-5 relative, elementwise (north_star; temperatures are bounded away from 0).
Cross-variant results must be bitwise identical (coarsening does not change results,
PAPER.md:145, 295; all variants evaluate the same hs_cell()).
"""
import numpy as np
import pytest

import oracle
import synth
from tests._util import hotspot_window_block, rel_err

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = 1e-5


@pytest.fixture(scope="module")
def rg():
    import paper_conf_cgo_ivanovzdem24_b200 as m
    return m


def _run(rg, T, P, iters, coef, g):
    t = torch.from_numpy(T).cuda()
    p = torch.from_numpy(P).cuda()
    c = rg.coeffs(coef["k"], coef["rx"], coef["ry"], coef["rz"], coef["amb"])
    out = rg.rodinia_hotspot(t, p, iters, coeffs=c, g=g)
    torch.cuda.synchronize()
    return out.cpu().numpy()


def _coef32(coef):
    return {k: float(np.float32(v)) for k, v in coef.items()}


UNC = (1, 1, 1, 1, 1, 0, 0)
SHAPES = [(1, 1), (1, 37), (37, 1), (15, 17), (64, 64), (100, 131), (257, 515), (128, 260)]


@pytest.mark.parametrize("R,C", SHAPES)
def test_uncoarsened_vs_oracle(rg, R, C):
    T, P = synth.hotspot_inputs(R, C)
    coef = _coef32(oracle.hotspot_coeffs_rodinia(512, 512, 0.016, 0.016))
    for iters in (0, 1, 2, 7):
        got = _run(rg, T, P, iters, coef, UNC)
        ref = oracle.hotspot(T, P, iters, **coef)
        assert rel_err(got, ref) <= TOL, (R, C, iters)


def test_config_c1_64x64_two_iterations(rg):
    # BASELINE configs[0]: 64x64, 2 iterations, h=1, coarsening 1x1, literal 16 mm chip.
    T, P = synth.hotspot_inputs(64, 64)
    coef = _coef32(oracle.hotspot_coeffs_rodinia(64, 64, 0.016, 0.016))
    got = _run(rg, T, P, 2, coef, UNC)
    assert rel_err(got, oracle.hotspot(T, P, 2, **coef)) <= TOL
    # the library's own coefficient helper agrees with the oracle's to fp32 rounding
    c = rg.rodinia_hotspot_coeffs_rodinia(64, 64)
    for k in ("k", "rx", "ry", "rz", "amb"):
        assert getattr(c, k) == np.float32(coef[k])


def _direct_grans():
    out = []
    for tx, ty in [(1, 1), (1, 2), (2, 1), (2, 2), (4, 1), (4, 4), (8, 1), (8, 2), (16, 1), (1, 16), (2, 8)]:
        for mode in (0, 1):
            for bx, by in [(1, 1), (3, 2), (7, 1)]:
                out.append((tx, ty, bx, by, 1, mode, 0))
    return out


def _stream_grans(rg):
    # every instantiated stream variant; the ptxas-pruned (spilling) ones through RODINIA_FORCE
    out = []
    for r in rg.rodinia_variants("hotspot"):
        g = r["g"]
        if not (g[6] & rg.RODINIA_STREAM):
            continue
        fl = g[6] | (rg.RODINIA_FORCE if r["status"] != 0 else 0)
        for bx, by in [(1, 1), (3, 2), (2, 16)]:
            out.append((g[0], 1, bx, by, g[4], 1, fl))
    return out


@pytest.mark.parametrize("R,C", [(200, 300), (61, 45), (33, 260)])
def test_all_variants_bit_identical(rg, R, C):
    T, P = synth.hotspot_inputs(R, C, seed_t=3, seed_p=4)
    coef = _coef32(oracle.hotspot_coeffs_rodinia(512, 512, 0.016, 0.016))
    iters = 17  # not a multiple of any temporal depth: exercises the remainder launches
    base = _run(rg, T, P, iters, coef, UNC)
    assert rel_err(base, oracle.hotspot(T, P, iters, **coef)) <= TOL
    for g in _direct_grans() + _stream_grans(rg):
        got = _run(rg, T, P, iters, coef, g)
        assert np.array_equal(got, base), g


def test_pins_on_gpu(rg):
    # ambient fixed point (bit-exact) and steady state (uniform grid unchanged)
    T = np.full((96, 160), 80.0, np.float32)
    Z = np.zeros_like(T)
    coef = {"k": 0.341333, "rx": 0.1, "ry": 0.1, "rz": 1 / 5120, "amb": 80.0}
    for g in (UNC, (4, 1, 4, 16, 8, 1, 2)):
        assert np.array_equal(_run(rg, T, Z, 40, coef, g), T)
    T = np.full((96, 160), 330.0, np.float32)
    Pss = np.full_like(T, np.float32((330.0 - 80.0) * np.float32(1 / 5120)))
    out = _run(rg, T, Pss, 40, coef, (4, 1, 4, 16, 8, 1, 2))
    assert rel_err(out, T) <= 1e-6


def test_full_size_windows_vs_oracle(rg):
    # BASELINE configs[2] at full size (16384^2, 1000 iterations, 512-grid coefficients) in the
    # launch configuration bench.py times: the TDO winner of the same rodinia_tune call (it is
    # also what a NULL granularity resolves to afterwards).  Three 64 x 64 output windows -- the
    # grid corner, a bottom-edge strip and the interior -- are compared elementwise with the
    # windowed fp64 oracle (cone radius 1001, OpenMP build over the host cores); the whole
    # output is compared bitwise with the uncoarsened variant over 24 steps.
    N, n = 16384, 1000
    T, P = synth.hotspot_inputs(N, N)
    coef = _coef32(oracle.hotspot_coeffs_rodinia(N, N, N * 31.25e-6, N * 31.25e-6))
    g, _ = rg.rodinia_tune("hotspot", N, N, n, nranks=1, reps=2)
    assert rg.rodinia_resolve("hotspot", N, N, n).astuple() == g.astuple()
    t = torch.from_numpy(T).cuda()
    p = torch.from_numpy(P).cuda()
    c = rg.coeffs(coef["k"], coef["rx"], coef["ry"], coef["rz"], coef["amb"])
    a = rg.rodinia_hotspot(t, p, 24, coeffs=c, g=g)
    b = rg.rodinia_hotspot(t, p, 24, coeffs=c, g=UNC)
    assert torch.equal(a, b), g.astuple()
    out = rg.rodinia_hotspot(t, p, n, coeffs=c, g=None).cpu().numpy()
    assert np.isfinite(out).all()
    oracle.set_threads(0)
    try:
        for (i0, j0) in [(0, 0), (N - 64, 8000), (8191, 12000)]:
            ref = hotspot_window_block(T, P, i0, j0, 64, 64, n, coef)
            got = out[i0:i0 + 64, j0:j0 + 64]
            assert rel_err(got, ref) <= TOL, (g.astuple(), i0, j0, rel_err(got, ref))
    finally:
        oracle.set_threads(1)


def test_host_entry_point(rg):
    T, P = synth.hotspot_inputs(130, 250)
    coef = _coef32(oracle.hotspot_coeffs_rodinia(512, 512, 0.016, 0.016))
    c = rg.coeffs(coef["k"], coef["rx"], coef["ry"], coef["rz"], coef["amb"])
    got = rg.rodinia_hotspot_host(T, P, 9, coeffs=c, g=(4, 1, 4, 2, 4, 1, 2))
    assert rel_err(got, oracle.hotspot(T, P, 9, **coef)) <= TOL


def test_variant_stats_match_runtime_attributes(rg):
    # the compile-time (ptxas) table agrees with cudaFuncGetAttributes through occupancy
    rows = rg.rodinia_variants("hotspot")
    assert rows and all(r["regs"] > 0 for r in rows)
    assert all(r["ctas_per_sm"] >= 1 for r in rows if r["status"] == 0)


def test_host_batch_pipelined_equals_single_calls(rg):
    # rodinia_hotspot_host_batch overlaps copies with solves (two device buffer sets): every
    # problem's result is bitwise the single-call result; 3 problems exercise set reuse
    c = rg.rodinia_hotspot_coeffs_rodinia(200, 300, 200 * 31.25e-6, 300 * 31.25e-6)
    ins = [synth.hotspot_inputs(200, 300, seed_t=10 + i, seed_p=20 + i) for i in range(3)]
    g = (4, 1, 1, 2, 8, 1, rg.RODINIA_STREAM)
    outs = rg.rodinia_hotspot_host_batch([t for t, _ in ins], [p for _, p in ins], 19, coeffs=c, g=g)
    for (t, p), o in zip(ins, outs):
        assert np.array_equal(o, rg.rodinia_hotspot_host(t, p, 19, coeffs=c, g=g))
