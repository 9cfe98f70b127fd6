"""GPU parity of pathfinder: bit-exact against the oracle for every variant (int32 DP)."""
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


def _run(rg, wall, g):
    w = torch.from_numpy(wall).cuda()
    out = rg.rodinia_pathfinder(w, g=g)
    torch.cuda.synchronize()
    return out.cpu().numpy()


SHAPES = [(1, 1), (1, 50), (2, 1), (7, 3), (5, 300), (30, 257), (100, 1000), (64, 4099)]


@pytest.mark.parametrize("R,C", SHAPES)
def test_uncoarsened_bit_exact(rg, R, C):
    wall = synth.pathfinder_wall(R, C)
    ref = oracle.pathfinder(wall)
    for h in (1, 2, 20):
        assert np.array_equal(_run(rg, wall, (1, 1, 1, 1, h, 0, 0)), ref), (R, C, h)


def test_all_variants_bit_exact(rg):
    wall = synth.pathfinder_wall(41, 3001, seed=4)
    ref = oracle.pathfinder(wall)
    for t in range(1, 9):
        for mode in (0, 1):
            for b in (1, 2):
                for h in (1, 3, 8, 20, 40, 1000):
                    g = (t, 1, b, 1, h, mode, 0)
                    try:
                        got = _run(rg, wall, g)
                    except rg.RodiniaError as e:
                        # a pyramid wider than the band, or a combination not instantiated
                        assert e.status in (rg.RODINIA_E_ILLEGAL_FACTOR, rg.RODINIA_E_NOT_BUILT), g
                        continue
                    assert np.array_equal(got, ref), g


def test_config_100000x100_sweep(rg):
    # BASELINE configs[1]: 100 rows x 100000 cols int32, thread-coarsening sweep 1..8, bit-exact
    wall = synth.pathfinder_wall(100, 100000)
    ref = oracle.pathfinder(wall)
    for t in range(1, 9):
        for g in [(t, 1, 1, 1, 20, 1, 0), (t, 1, 1, 1, 99, 1, 0), (t, 1, 1, 1, 8, 0, 0)]:
            try:
                got = _run(rg, wall, g)
            except rg.RodiniaError as e:
                assert e.status == rg.RODINIA_E_ILLEGAL_FACTOR, g
                continue
            assert np.array_equal(got, ref), g
    assert np.array_equal(_run(rg, wall, None), ref)  # default / tuned


def test_faithful_mode_rejects_non_divisors(rg):
    wall = synth.pathfinder_wall(10, 500)
    for t in (3, 5, 6, 7):
        with pytest.raises(rg.RodiniaError) as e:
            _run(rg, wall, (t, 1, 1, 1, 4, 1, rg.RODINIA_FAITHFUL))
        assert e.value.status == rg.RODINIA_E_ILLEGAL_FACTOR
    ref = oracle.pathfinder(wall)
    for t in (1, 2, 4, 8):
        assert np.array_equal(_run(rg, wall, (t, 1, 1, 1, 4, 1, rg.RODINIA_FAITHFUL)), ref)


def test_constant_wall_and_host_entry(rg):
    wall = np.full((100, 3000), 7, np.int32)
    assert np.all(_run(rg, wall, (4, 1, 1, 1, 20, 1, 0)) == 700)
    w2 = synth.pathfinder_wall(33, 777)
    assert np.array_equal(rg.rodinia_pathfinder_host(w2, g=(2, 1, 1, 1, 5, 1, 0)), oracle.pathfinder(w2))


def test_tuner_returns_legal_bit_exact_choice(rg):
    best, rows = rg.rodinia_tune("pathfinder", 100, 100000, 1, reps=2)
    assert any(r["status"] == 0 and r["median_ms"] > 0 for r in rows)
    wall = synth.pathfinder_wall(100, 100000)
    assert np.array_equal(_run(rg, wall, best), oracle.pathfinder(wall))


def test_unaligned_views_bit_exact(rg):
    # offset views of the wall and result (4 bytes off 16-byte alignment) take the scalar edge
    # path of the warp-band kernel instead of faulting on 128-bit accesses
    R, C = 60, 4096
    wall = synth.pathfinder_wall(R, C, seed=8)
    ref = oracle.pathfinder(wall)
    wb = torch.zeros(R * C + 1, dtype=torch.int32, device="cuda")
    w = wb[1:].view(R, C)
    w.copy_(torch.from_numpy(wall))
    ob = torch.zeros(C + 3, dtype=torch.int32, device="cuda")
    for g in [(4, 1, 1, 1, 20, 1, 2), (2, 1, 1, 1, 12, 1, 2), (8, 1, 1, 1, 16, 1, 2)]:
        out = rg.rodinia_pathfinder(w, g=g, out=ob[1:1 + C])
        torch.cuda.synchronize()
        assert np.array_equal(out.cpu().numpy(), ref), g
        aligned = rg.rodinia_pathfinder(torch.from_numpy(wall).cuda(), g=g)
        assert np.array_equal(aligned.cpu().numpy(), ref), g
