"""Pins for the hotspot3D oracle (CPU only): closed-form coefficients, the ambient fixed point,
3-D cosine eigenmodes of the clamped 7-point operator, the discrete heat balance, mirror
symmetry and reduction of a z-uniform field to nz = 1."""
import numpy as np
import pytest

import oracle


def test_coeffs_closed_form():
    # sdc = dt/Cap = PRECISION/(MAX_PD dx dy); 1/Rx = 2 K t dx/dy; 1/Ry = 2 K t dy/dx;
    # 1/Rz = K dx dy / dz; cc = 1 - (2ce + 2cn + 3ct)   (Rodinia 512 x 512 x 8 chip)
    nx = ny = 512
    nz = 8
    c = oracle.hotspot3d_coeffs(nx, ny, nz)
    dx, dy, dz = 0.016 / ny, 0.016 / nx, 0.0005 / nz
    sdc = 1e-3 / (3e6 * dx * dy)
    assert c["sdc"] == pytest.approx(sdc, rel=1e-13)
    assert c["ce"] == pytest.approx(sdc * 2 * 100 * 0.0005 * dx / dy, rel=1e-13)
    assert c["cn"] == pytest.approx(sdc * 2 * 100 * 0.0005 * dy / dx, rel=1e-13)
    assert c["ct"] == pytest.approx(sdc * 100 * dx * dy / dz, rel=1e-13)
    assert c["cc"] == pytest.approx(1 - (2 * c["ce"] + 2 * c["cn"] + 3 * c["ct"]), rel=1e-14)
    assert c["cw"] == c["ce"] and c["cs"] == c["cn"] and c["cb"] == c["ct"]
    assert c["sdc"] == pytest.approx(0.3413333, rel=1e-6)


def test_ambient_fixed_point():
    c = oracle.hotspot3d_coeffs(16, 12, 5)
    t = np.full((5, 12, 16), 80.0)
    out = oracle.hotspot3d(t, np.zeros_like(t), 20, c)
    np.testing.assert_allclose(out, t, rtol=1e-14)


@pytest.mark.parametrize("shape,mode", [((6, 10, 14), (2, 3, 1)), ((1, 9, 7), (0, 1, 4)), ((8, 1, 5), (3, 0, 2))])
def test_cosine_eigenmode(shape, mode):
    # u = T - amb, P = 0: each clamped direction has eigenvectors cos(pi m (i + 1/2)/n) with
    # cos-shift 2 cos(pi m/n); the step multiplies the mode by
    #   g = cc + 2 ce cos(pi mx/nx) + 2 cn cos(pi my/ny) + 2 ct cos(pi mz/nz)
    # (distinct ce, cn, ct: a rectangular chip with nz layers)
    nz, ny, nx = shape
    mz, my, mx = mode
    c = oracle.hotspot3d_coeffs(nx, ny, nz, 0.016, 0.011, 0.0007)
    z = (np.arange(nz) + 0.5) / nz
    y = (np.arange(ny) + 0.5) / ny
    x = (np.arange(nx) + 0.5) / nx
    u = np.cos(np.pi * mz * z)[:, None, None] * np.cos(np.pi * my * y)[None, :, None] * np.cos(np.pi * mx * x)[None, None, :]
    t0 = c["amb"] + 3.0 * u
    n = 15
    out = oracle.hotspot3d(t0, np.zeros_like(t0), n, c)
    g = c["cc"] + 2 * c["ce"] * np.cos(np.pi * mx / nx) + 2 * c["cn"] * np.cos(np.pi * my / ny) + \
        2 * c["ct"] * np.cos(np.pi * mz / nz)
    np.testing.assert_allclose(out - c["amb"], g ** n * 3.0 * u, rtol=0, atol=1e-11)


def test_heat_balance():
    rng = np.random.default_rng(3)
    c = oracle.hotspot3d_coeffs(11, 9, 4)
    t = 300 + 30 * rng.random((4, 9, 11))
    p = rng.random((4, 9, 11))
    out = oracle.hotspot3d(t, p, 1, c)
    rhs = c["sdc"] * p.sum() + c["ct"] * np.sum(c["amb"] - t)
    assert out.sum() - t.sum() == pytest.approx(rhs, rel=1e-9)


def test_mirror_symmetry():
    rng = np.random.default_rng(4)
    c = oracle.hotspot3d_coeffs(13, 10, 6)
    t = 300 + 30 * rng.random((6, 10, 13))
    p = rng.random((6, 10, 13))
    base = oracle.hotspot3d(t, p, 5, c)
    for ax in range(3):
        got = oracle.hotspot3d(np.flip(t, ax), np.flip(p, ax), 5, c)
        np.testing.assert_allclose(got, np.flip(base, ax), rtol=1e-14)


def test_z_uniform_reduces_to_one_layer():
    # identical layers: B = T = c in effect, so every layer evolves like the nz = 1 problem
    # with the same coefficients
    rng = np.random.default_rng(5)
    c = oracle.hotspot3d_coeffs(12, 8, 4)
    layer = 300 + 30 * rng.random((1, 8, 12))
    pl = rng.random((1, 8, 12))
    one = oracle.hotspot3d(layer, pl, 6, c)
    many = oracle.hotspot3d(np.repeat(layer, 4, 0), np.repeat(pl, 4, 0), 6, c)
    np.testing.assert_allclose(many, np.repeat(one, 4, 0), rtol=1e-14)
