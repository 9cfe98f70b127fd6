"""Heuristic pre-pruning model (PAPER.md:253-265 kernel statistics, 405):
host-only checks of rodinia_model_ms against closed forms and the orderings the work counts
fix.  The GPU tests (test_gpu_tune.py) check that pruned tuning finds a variant within a few
percent of full timing-driven tuning."""
import math

import pytest

import paper_conf_cgo_ivanovzdem24_b200 as rg

STREAM = rg.RODINIA_STREAM
N = 16384
HBM = 6.45e12     # model's nominal sustained HBM B/s without a device (model.cu ModelDevice)


def _m(kernel, g, **kw):
    return rg.rodinia_model_ms(kernel, g, **kw)


def _nodev():
    import torch
    return not torch.cuda.is_available()


@pytest.mark.skipif(not _nodev(), reason="closed form uses the nominal B200 constants (no device)")
def test_direct_hotspot_is_the_hbm_roofline():
    # float4 contiguous variant, 256 threads, enough warps: HBM-bound at 12 B per cell-update
    ms = _m("hotspot", (4, 1, 1, 1, 1, 1, 0), rows=N, cols=N, iterations=10, regs=40, threads=64,
            ctas_per_sm=16)
    waves = (N // 16) ** 2 / (16 * 148)
    hide = 1 - math.exp(-2 * 32 / 32)   # 16 CTAs x 2 warps against W_sat = 32
    t_hbm = 10 * 12.0 * N * N / HBM * 1e3 * (math.ceil(waves) / waves) / hide + 10 * 2.5e-3
    assert ms == pytest.approx(t_hbm, rel=1e-4)


@pytest.mark.skipif(not _nodev(), reason="closed form uses the nominal B200 constants (no device)")
def test_stream_hotspot_closed_form():
    # V=4, H=8, chunk 128 rows, 12 warps/SM: max(bytes/BW, instructions/issue) + launches
    V, H, chunk, it = 4, 8, 128, 16
    cells = N * N
    col = 32 * V / (32 * V - 2 * H)
    # a quarter of the staged halo re-reads reach HBM (model.cu l2_absorbed)
    bytes_ = (it // H) * cells * (8 * (1 + 0.27 * (col * (chunk + 2 * H + 8) / chunk - 1)) + 4)
    instr = (it // H) * cells * H * col * (chunk + H - 1) / chunk * 6.4
    ctas = math.ceil(N / (32 * V - 2 * H)) * (N // chunk)
    waves = ctas / (12 * 148)
    hide = 1 - math.exp(-2 * 12 / 8)    # 12 one-warp CTAs against W_sat = 8
    t = max(bytes_ / HBM, instr / (148 * 128 * 1.965e9)) * math.ceil(waves) / waves / hide + (it // H) * 2.5e-6
    ms = _m("hotspot", (V, 1, 1, chunk // 16, H, 1, STREAM | (12 << 8)), rows=N, cols=N, iterations=it,
            regs=162, threads=32, ctas_per_sm=12)
    assert ms == pytest.approx(t * 1e3, rel=1e-3)


def test_temporal_blocking_beats_one_step_per_launch():
    direct = _m("hotspot", (1, 1, 1, 1, 1, 0, 0), rows=N, cols=N, iterations=1000, regs=20, threads=256)
    stream = _m("hotspot", (4, 1, 1, 8, 8, 1, STREAM | (12 << 8)), rows=N, cols=N, iterations=1000,
                regs=162, threads=32)
    assert direct > 0 and stream > 0
    assert direct / stream > 3.0


def test_wave_quantization():
    # 4.27 waves of CTAs take 5 wave times; 8.54 take 9
    kw = dict(rows=N, cols=N, iterations=1000, regs=168, threads=32, ctas_per_sm=10)
    t12 = _m("hotspot", (4, 1, 1, 12, 8, 1, STREAM | (10 << 8)), **kw)
    t24 = _m("hotspot", (4, 1, 1, 24, 8, 1, STREAM | (10 << 8)), **kw)
    assert t24 > t12


def test_halo_redundancy_orders_chunk_heights():
    # shorter chunks recompute the temporal halo more often
    kw = dict(rows=N, cols=N, iterations=96, regs=162, threads=32, ctas_per_sm=12)
    t = [_m("hotspot", (4, 1, 1, by, 8, 1, STREAM | (12 << 8)), **kw) for by in (1, 2, 4, 8)]
    assert t == sorted(t, reverse=True) and t[0] > 1.2 * t[-1]


def test_occupancy_and_spills_penalise():
    base = dict(rows=N, cols=N, iterations=10, threads=256)
    lo = _m("hotspot", (1, 1, 1, 1, 1, 0, 0), regs=32, **base)        # 8 CTAs = 64 warps/SM
    hi = _m("hotspot", (1, 1, 1, 1, 1, 0, 0), regs=255, **base)       # 1 CTA = 8 warps/SM
    sp = _m("hotspot", (1, 1, 1, 1, 1, 0, 0), regs=32, spill_bytes=64, **base)
    assert hi > 2 * lo
    assert sp > lo


def test_sub_warp_ctas_waste_lanes():
    # (16,16) thread coarsening leaves one thread per CTA: 1/32 of every warp-instruction useful
    full = _m("hotspot", (1, 1, 1, 1, 1, 0, 0), rows=N, cols=N, iterations=10, regs=32, threads=256)
    tiny = _m("hotspot", (16, 2, 1, 1, 1, 0, 0), rows=N, cols=N, iterations=10, regs=64, threads=8)
    assert tiny > full


def test_srad_families_order():
    kw = dict(rows=8192, cols=8192, iterations=100)
    dataflow = _m("srad", (1, 1, 1, 1, 1, 0, 0), regs=30, threads=256, **kw)
    fused = _m("srad", (1, 1, 1, 1, 1, 1, 0), regs=40, threads=256, smem_bytes=2500, **kw)
    stream = _m("srad", (4, 1, 1, 3, 1, 1, STREAM), regs=120, threads=32, **kw)
    assert dataflow > fused > stream > 0
    # Rodinia dataflow: 52 B per update is a hard lower bound of its estimate
    assert dataflow >= 100 * 52.0 * 8192 * 8192 / 8.2e12 * 1e3


def _stats(kernel, g):
    for r in rg.rodinia_variants(kernel):
        if tuple(r["g"]) == tuple(g):
            return dict(regs=r["regs"], threads=r["threads"], smem_bytes=max(r["smem_bytes"], 0))
    raise KeyError(g)


def test_hotspot3d_plane_beats_direct():
    # with the build's own ptxas statistics (48 registers -> 40 warps/SM for Rodinia's shape)
    kw = dict(rows=1024, cols=1024, depth=64, iterations=10)
    gd, gp = (1, 1, 1, 1, 1, 0, 0), (2, 2, 1, 1, 1, 1, STREAM)
    d = _m("hotspot3d", gd, **_stats("hotspot3d", gd), **kw)
    p = _m("hotspot3d", gp, **_stats("hotspot3d", gp), **kw)
    assert d > p > 0


def test_unmodelled_workloads_and_errors():
    assert _m("lud", (4, 2, 2, 2, 1, 1, 0), rows=1024, cols=1024, iterations=16, regs=64, threads=64) == -1
    assert _m("pathfinder", (4, 1, 1, 1, 20, 1, 0), rows=100, cols=100000, regs=40, threads=64) == -1
    with pytest.raises(rg.RodiniaError):
        _m("hotspot", (0, 1, 1, 1, 1, 0, 0), rows=N, cols=N)
    with pytest.raises(rg.RodiniaError):
        _m("hotspot", (1, 1, 1, 1, 1, 0, 0), rows=0, cols=N)


def test_tune_pruned_argument_validation():
    import ctypes
    import torch
    p = rg.Problem(256, 256, 16, 1, 0, 0)
    best = rg.Granularity()
    n = ctypes.c_int32(0)
    # bad arguments are rejected before any device work
    assert rg.lib.rodinia_tune_pruned(0, None, 1, 4, ctypes.byref(best), None, ctypes.byref(n)) == rg.RODINIA_E_INVALID
    assert rg.lib.rodinia_tune_pruned(0, ctypes.byref(p), 0, 4, ctypes.byref(best), None, ctypes.byref(n)) == rg.RODINIA_E_INVALID
    assert rg.lib.rodinia_tune_pruned(9, ctypes.byref(p), 1, 4, ctypes.byref(best), None, ctypes.byref(n)) == rg.RODINIA_E_INVALID
    if not torch.cuda.is_available():
        st = rg.lib.rodinia_tune_pruned(0, ctypes.byref(p), 1, 4, ctypes.byref(best), None, ctypes.byref(n))
        assert st == rg.RODINIA_E_NODEV
