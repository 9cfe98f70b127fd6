"""Pins for oracle.hotspot / oracle.hotspot_coeffs_rodinia (CPU only).

None of these re-types the oracle's stencil: each checks it against something the
mathematics fixes independently -- algebraically simplified coefficient formulas, the
scalar recurrence of a uniform field, the closed-form decay of the clamped-Laplacian
cosine eigenmodes, the discrete heat balance, exact mirror symmetry, and a hand-checked
fixture (tests/golden/hotspot_mini.txt).
"""
import os

import numpy as np
import pytest

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def test_coeffs_closed_form_square_chip():
    # Algebra on the Rodinia constants (H1):
    #   k = step/Cap = PRECISION / (MAX_PD * gw * gh) = 1e-3 / (3e6 * gw * gh)
    #   rx = 1/Rx = 2*K_SI*t_chip*gh/gw = 0.1*gh/gw ; ry = 0.1*gw/gh
    #   rz = 1/Rz = K_SI*gw*gh/t_chip = 2e5*gw*gh
    c = oracle.hotspot_coeffs_rodinia(64, 64, 0.016, 0.016)
    gw = gh = 0.016 / 64
    assert c["k"] == pytest.approx(1e-3 / (3e6 * gw * gh), rel=1e-14)
    assert c["k"] == pytest.approx(0.005333333333333333, rel=1e-12)
    assert c["rx"] == pytest.approx(0.1, rel=1e-14)
    assert c["ry"] == pytest.approx(0.1, rel=1e-14)
    assert c["rz"] == pytest.approx(0.0125, rel=1e-14)
    assert c["amb"] == 80.0


def test_coeffs_512_cell_size():
    # The benchmark's 16384^2 grid uses the 512-grid cell size (chip = N * 31.25 um),
    # DESIGN.md H1: k = 0.341333.., rx = ry = 0.1, rz = 1/5120.
    n = 16384
    c = oracle.hotspot_coeffs_rodinia(n, n, n * 31.25e-6, n * 31.25e-6)
    assert c["k"] == pytest.approx(0.3413333333333333, rel=1e-12)
    assert c["rx"] == pytest.approx(0.1, rel=1e-13)
    assert c["rz"] == pytest.approx(1 / 5120, rel=1e-12)


def test_coeffs_rectangular_cells_not_transposed():
    c = oracle.hotspot_coeffs_rodinia(64, 64, 0.016, 0.008)  # gw = 2.5e-4, gh = 1.25e-4
    gw, gh = 0.016 / 64, 0.008 / 64
    assert c["rx"] == pytest.approx(0.1 * gh / gw, rel=1e-14)  # 0.05
    assert c["ry"] == pytest.approx(0.1 * gw / gh, rel=1e-14)  # 0.2
    assert c["rz"] == pytest.approx(2e5 * gw * gh, rel=1e-14)
    assert c["k"] == pytest.approx(1e-3 / (3e6 * gw * gh), rel=1e-14)


def test_ambient_fixed_point_bit_exact():
    t = np.full((13, 17), 80.0)
    out = oracle.hotspot(t, np.zeros_like(t), 25, 0.3, 0.1, 0.1, 0.01, 80.0)
    assert np.array_equal(out, t)


def test_uniform_field_scalar_recurrence():
    # Uniform T, uniform P: neighbour terms vanish, u = T - amb obeys
    # u' = u + k (P - rz u)  =>  u_n = u_inf + (u_0 - u_inf)(1 - k rz)^n, u_inf = P/rz.
    k, rx, ry, rz, amb, p, t0, n = 0.34, 0.1, 0.1, 0.05, 80.0, 0.2, 330.0, 40
    out = oracle.hotspot(np.full((9, 11), t0), np.full((9, 11), p), n, k, rx, ry, rz, amb)
    u_inf = p / rz
    expect = amb + u_inf + (t0 - amb - u_inf) * (1 - k * rz) ** n
    np.testing.assert_allclose(out, expect, rtol=1e-13)


def test_steady_state_unchanged():
    # T = T0, P = (T0 - amb) rz is a fixed point (the north star's uniform steady grid).
    k, rz, amb, t0 = 0.341333, 1 / 5120, 80.0, 330.0
    t = np.full((16, 16), t0)
    out = oracle.hotspot(t, np.full_like(t, (t0 - amb) * rz), 100, k, 0.1, 0.1, rz, amb)
    np.testing.assert_allclose(out, t, rtol=1e-15, atol=0)


@pytest.mark.parametrize("R,C,m,q", [(24, 40, 3, 2), (17, 9, 1, 4), (1, 33, 5, 0), (20, 1, 0, 7)])
def test_cosine_eigenmode_closed_form(R, C, m, q):
    # With the clamped (Neumann) boundary, v_j = cos(pi m (j + 1/2) / C) is an eigenvector of
    # (E + W - 2c) with eigenvalue -4 sin^2(pi m / 2C).  For P = 0:
    #   T_n - amb = g^n (T_0 - amb),  g = 1 - k (4 rx sin^2(pi m/2C) + 4 ry sin^2(pi q/2R) + rz)
    # rx != ry and R != C so a transposed coefficient or index fails.
    k, rx, ry, rz, amb, n = 0.2, 0.13, 0.37, 0.01, 80.0, 30
    jj = (np.arange(C) + 0.5) / C
    ii = (np.arange(R) + 0.5) / R
    mode = np.outer(np.cos(np.pi * q * ii), np.cos(np.pi * m * jj))
    t0 = amb + 5.0 * mode
    out = oracle.hotspot(t0, np.zeros_like(t0), n, k, rx, ry, rz, amb)
    g = 1 - k * (4 * rx * np.sin(np.pi * m / (2 * C)) ** 2 + 4 * ry * np.sin(np.pi * q / (2 * R)) ** 2 + rz)
    np.testing.assert_allclose(out - amb, g ** n * (t0 - amb), rtol=0, atol=1e-12 * 5)


def test_heat_balance():
    # The clamped Laplacian sums to zero, so sum(T') - sum(T) = k * sum(P + (amb - T) rz).
    rng = np.random.default_rng(0)
    t = 300 + 30 * rng.random((31, 23))
    p = rng.random((31, 23))
    k, rz, amb = 0.3, 0.07, 80.0
    out = oracle.hotspot(t, p, 1, k, 0.1, 0.2, rz, amb)
    lhs = out.sum() - t.sum()
    rhs = k * np.sum(p + (amb - t) * rz)
    assert lhs == pytest.approx(rhs, rel=1e-9)


def test_mirror_symmetry_bit_exact():
    rng = np.random.default_rng(1)
    t = 300 + 30 * rng.random((19, 26))
    p = rng.random((19, 26))
    args = (7, 0.3, 0.1, 0.2, 0.01, 80.0)
    base = oracle.hotspot(t, p, *args)
    assert np.array_equal(oracle.hotspot(t[::-1], p[::-1], *args), base[::-1])
    assert np.array_equal(oracle.hotspot(t[:, ::-1], p[:, ::-1], *args), base[:, ::-1])


def test_row_translation_invariance_reduces_to_1d():
    # Rows identical => N = S = c, so every row evolves like the 1 x C problem.
    rng = np.random.default_rng(2)
    row = 300 + 30 * rng.random(29)
    prow = rng.random(29)
    args = (5, 0.3, 0.1, 0.2, 0.01, 80.0)
    one = oracle.hotspot(row[None, :], prow[None, :], *args)
    many = oracle.hotspot(np.tile(row, (6, 1)), np.tile(prow, (6, 1)), *args)
    assert np.array_equal(many, np.tile(one, (6, 1)))


def _load_golden(name):
    blocks, cur = {}, None
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            if line.startswith("[") and line.endswith("]"):
                cur = line[1:-1]
                blocks[cur] = []
            else:
                blocks[cur].append([float(x) for x in line.split()])
    return {k: np.array(v) for k, v in blocks.items()}


def test_hand_checked_mini_case():
    g = _load_golden("hotspot_mini.txt")
    k, rx, ry, rz, amb = g["coeffs"][0]
    out = oracle.hotspot(g["t0"], np.zeros_like(g["t0"]), 1, k, rx, ry, rz, amb)
    assert np.array_equal(out, g["t1"])


def test_zero_iterations_copies_and_bad_args():
    t = np.arange(12.0).reshape(3, 4)
    assert np.array_equal(oracle.hotspot(t, t, 0, 1, 1, 1, 1), t)
    with pytest.raises(oracle.OracleError):
        oracle.hotspot(t, t, -1, 1, 1, 1, 1)
