"""C-ABI tests that need no GPU: the library loads, exports every symbol the header
declares, validates arguments before any CUDA call, and the compile-time filter's ptxas
parser / pruning rules behave as the paper describes."""
import ctypes
import os
import re
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))

import oracle  # noqa: E402
import paper_conf_cgo_ivanovzdem24_b200 as rg  # noqa: E402
import ptxas_filter  # noqa: E402


def _header_functions():
    txt = open(os.path.join(ROOT, "include", "rodinia_gran.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(rodinia_\w+)\s*\(", txt)))


def test_every_header_symbol_exported():
    names = _header_functions()
    assert len(names) >= 20
    for n in names:
        assert hasattr(rg.lib, n), n
    assert set(names) == set(rg.EXPORTED)
    assert rg.lib.rodinia_abi_version() == 3


def test_status_strings():
    assert rg.status_string(rg.RODINIA_E_FILTERED) == "RODINIA_E_FILTERED"
    assert rg.status_string(0) == "RODINIA_OK"


def _hs(tin=1, p=2, tout=3, R=8, C=8, it=1, g=None, coef=None):
    return rg.lib.rodinia_hotspot(ctypes.c_void_p(tin), ctypes.c_void_p(p), ctypes.c_void_p(tout),
                                  None, R, C, it, coef, rg._g(g), None)


def test_hotspot_argument_validation_without_device():
    assert _hs(tin=0) == rg.RODINIA_E_INVALID
    assert _hs(R=0) == rg.RODINIA_E_INVALID
    assert _hs(it=-1) == rg.RODINIA_E_INVALID
    assert _hs(tout=1) == rg.RODINIA_E_INVALID  # aliasing
    bad = rg.HotspotCoeffs(float("nan"), 0.1, 0.1, 0.1, 80)
    assert _hs(coef=ctypes.byref(bad)) == rg.RODINIA_E_INVALID
    assert _hs(g=(3, 1, 1, 1, 1, 0, 0)) == rg.RODINIA_E_ILLEGAL_FACTOR  # 3 does not divide 16
    assert _hs(g=(1, 1, 0, 1, 1, 0, 0)) == rg.RODINIA_E_ILLEGAL_FACTOR
    assert _hs(g=(1, 1, 1, 1, 4, 0, 0)) == rg.RODINIA_E_ILLEGAL_FACTOR  # temporal needs STREAM
    assert _hs(g=(4, 1, 1, 1, 5, 1, 2)) == rg.RODINIA_E_NOT_BUILT
    # arbitrary (even prime) block factors are legal; on a host without a GPU
    # the call then reports NODEV
    import torch
    st = _hs(g=(1, 1, 7, 3, 1, 0, 0))
    assert st == (rg.RODINIA_OK if torch.cuda.is_available() else rg.RODINIA_E_NODEV) or torch.cuda.is_available()
    if not torch.cuda.is_available():
        assert "device" in rg.last_error().lower()


def test_coefficient_helper_matches_oracle():
    for (R, C, w, h) in [(64, 64, 0.016, 0.016), (16384, 16384, 0.512, 0.512), (64, 32, 0.016, 0.008)]:
        c = rg.rodinia_hotspot_coeffs_rodinia(R, C, w, h)
        o = oracle.hotspot_coeffs_rodinia(R, C, w, h)
        for k in ("k", "rx", "ry", "rz", "amb"):
            assert getattr(c, k) == np.float32(o[k]), (R, C, k)


def test_variants_listing_without_device():
    rows = rg.rodinia_variants("hotspot")
    assert len(rows) >= 40
    assert rows[0]["g"] == rg.UNCOARSENED
    for r in rows:
        assert r["regs"] > 0 and r["threads"] > 0
        if r["spill_bytes"] > 0:
            assert r["status"] == rg.RODINIA_E_FILTERED  # new spills are pruned
        else:
            assert r["status"] == rg.RODINIA_OK


def test_ptxas_parser_on_canned_log():
    text = open(os.path.join(ROOT, "tests", "golden", "ptxas_sample.log")).read()
    st = ptxas_filter.parse_ptxas_log(text)
    assert set(s.key for s in st.values()) == {
        "void rg::hs_direct<16, 2, 1>", "void rg::hs_direct<1, 1, 0>", "big_smem"}
    by = {s.key: s for s in st.values()}
    a = by["void rg::hs_direct<16, 2, 1>"]
    assert (a.regs, a.spill_stores, a.spill_loads, a.stack) == (64, 8, 12, 8)
    b = by["void rg::hs_direct<1, 1, 0>"]
    assert (b.regs, b.spill_stores, b.spill_loads) == (40, 0, 0)
    assert by["big_smem"].smem == 233472


def test_prune_rules():
    st = ptxas_filter.KernelStats("x", "x", regs=64, spill_stores=8, spill_loads=12)
    assert ptxas_filter.prune_reason(st, 8, base_spill=0) == "new-spill"
    assert ptxas_filter.prune_reason(st, 8, base_spill=4) is None       # not *new* spilling
    big = ptxas_filter.KernelStats("y", "y", regs=24, smem=233472)
    assert ptxas_filter.prune_reason(big, 256, base_spill=0) == "smem"  # > 227 KB
    fat = ptxas_filter.KernelStats("z", "z", regs=255)
    assert ptxas_filter.prune_reason(fat, 512, base_spill=0) == "occupancy"
    ok = ptxas_filter.KernelStats("w", "w", regs=40)
    assert ptxas_filter.prune_reason(ok, 256, base_spill=0) is None


def test_split_total_footnote_examples():
    # PAPER.md:189 (footnote 4): 16 -> (4, 2, 2), 6 -> (3, 2, 1)
    assert rg.rodinia_split_total(16, 3) == (4, 2, 2)
    assert rg.rodinia_split_total(6, 3) == (3, 2, 1)
    # 2-D and edge cases of the reading (largest prime to the smallest current factor)
    assert rg.rodinia_split_total(16, 2) == (4, 4)
    assert rg.rodinia_split_total(14, 2) == (7, 2)
    assert rg.rodinia_split_total(7, 3) == (7, 1, 1)
    assert rg.rodinia_split_total(1, 3) == (1, 1, 1)
    for t in range(1, 65):
        x, y, z = rg.rodinia_split_total(t, 3)
        assert x * y * z == t and max(x, y, z) <= t
    with pytest.raises(rg.RodiniaError):
        rg.rodinia_split_total(0, 3)


def test_hotspot_host_batch_argument_validation_without_device():
    null3 = (ctypes.c_void_p * 1)(None)
    ok = (ctypes.c_void_p * 1)(1)
    assert rg.lib.rodinia_hotspot_host_batch(ok, ok, ok, -1, 8, 8, 1, None, None, None) == rg.RODINIA_E_INVALID
    assert rg.lib.rodinia_hotspot_host_batch(null3, ok, ok, 1, 8, 8, 1, None, None, None) == rg.RODINIA_E_INVALID
    assert rg.lib.rodinia_hotspot_host_batch(ok, ok, ok, 1, 0, 8, 1, None, None, None) == rg.RODINIA_E_INVALID
    assert rg.lib.rodinia_hotspot_host_batch(None, None, None, 0, 8, 8, 1, None, None, None) == rg.RODINIA_OK


def _nodev_or_ok():
    import torch
    return rg.RODINIA_OK if torch.cuda.is_available() else rg.RODINIA_E_NODEV


def test_filter_enforced_at_the_boundary():
    # An explicit call naming an instantiation the compile-time ptxas filter pruned (new spills,
    # PAPER.md:267) is refused before any CUDA call; RODINIA_FORCE runs it anyway.  hotspot:
    # hs_stream<4, 4, 16> (V = 4, H = 4, OCC 16 -> <= 128 registers) spills in this build.
    S, F = rg.RODINIA_STREAM, rg.RODINIA_FORCE
    spilling = (4, 1, 1, 4, 4, 1, S | (16 << 8))
    rows = {r["g"]: r for r in rg.rodinia_variants("hotspot")}
    assert rows[spilling]["status"] == rg.RODINIA_E_FILTERED and rows[spilling]["spill_bytes"] > 0
    assert _hs(R=64, C=256, g=spilling) == rg.RODINIA_E_FILTERED
    assert "RODINIA_FORCE" in rg.last_error()
    if _nodev_or_ok() == rg.RODINIA_E_NODEV:  # past the filter the call needs a device
        assert _hs(R=64, C=256, g=spilling[:6] + (spilling[6] | F,)) == rg.RODINIA_E_NODEV
    # every pruned hotspot instantiation is refused, every surviving one passes the filter
    for g, r in rows.items():
        st = _hs(R=64, C=256, g=g)
        if r["status"] == rg.RODINIA_E_FILTERED:
            assert st == rg.RODINIA_E_FILTERED, g
        else:
            assert st != rg.RODINIA_E_FILTERED, g


def test_filter_enforced_lud_and_others():
    # lud: the pruned internal instantiations (panel 16 or 32; the listing's granularity does not
    # carry the panel width, so one of the two must refuse it)
    lud = lambda g, panel: rg.lib.rodinia_lud(ctypes.c_void_p(16), 256, panel, rg._g(g), None)
    pruned = [r["g"] for r in rg.rodinia_variants("lud") if r["status"] == rg.RODINIA_E_FILTERED]
    assert pruned
    for g in pruned:
        sts = {lud(g, 16), lud(g, 32)}
        assert rg.RODINIA_E_FILTERED in sts, g
        forced = g[:6] + (g[6] | rg.RODINIA_FORCE,)
        assert rg.RODINIA_E_FILTERED not in {lud(forced, 16), lud(forced, 32)}, g
    # srad / pathfinder / hotspot3d: nothing is pruned in this build; surviving variants pass
    for k in ("srad", "pathfinder", "hotspot3d"):
        for r in rg.rodinia_variants(k):
            assert r["status"] in (rg.RODINIA_OK, rg.RODINIA_E_FILTERED)
    sr = rg.lib.rodinia_srad(ctypes.c_void_p(16), 64, 64, 0, 9, 0, 9, ctypes.c_float(0.5), 2,
                             rg._g((4, 1, 1, 2, 1, 1, rg.RODINIA_STREAM)), None)
    assert sr == _nodev_or_ok()
