"""Pins for the srad_v2 oracle (CPU only).

Independent checks: closed-form q0sqr of a two-valued ROI, closed-form diffusion
coefficient of quadratic profiles (derived by hand, see comments), closed-form decay of
cosine eigenmodes when every c saturates at 1 (pure 5-point diffusion), the exact
one-iteration dependency footprint (pins the c(i+1,j) / c(i,j+1) indices), uniform and
lambda = 0 fixed points, the maximum principle and the multi-iteration dependency cone.
"""
import numpy as np
import pytest

import oracle


def test_two_valued_roi_q0sqr_closed_form():
    # half a, half b: mean = (a+b)/2, var = ((a-b)/2)^2 => q0sqr = ((a-b)/(a+b))^2
    a, b = 1.25, 2.5
    J = np.full((10, 12), 1.7)
    J[2:6, 3:5] = a
    J[2:6, 5:7] = b
    q = oracle.srad_q0sqr(J, 2, 5, 3, 6)
    assert q == pytest.approx(((a - b) / (a + b)) ** 2, rel=1e-14)


def test_degenerate_roi_mean_zero():
    J = np.zeros((4, 4))
    with pytest.raises(oracle.OracleError) as e:
        oracle.srad_q0sqr(J, 0, 1, 0, 1)
    assert e.value.code == oracle.EDEGENERATE


def test_bad_roi_rejected():
    J = np.ones((4, 4))
    for roi in [(0, 4, 0, 1), (2, 1, 0, 1), (-1, 1, 0, 1), (0, 1, 3, 4)]:
        with pytest.raises(oracle.OracleError):
            oracle.srad_q0sqr(J, *roi)


def _c_from_q(q, q0):
    t = 0.0 if q == q0 else (q - q0) / (q0 * (1 + q0))
    return min(1.0, max(0.0, 1 / (1 + t)))


@pytest.mark.parametrize("axis", [0, 1])
def test_coefficient_closed_form_quadratic_profile(axis):
    # J = K + x^2 along one axis, constant along the other.  At an interior x:
    #   the two differences are (x-1)^2 - x^2 = 1 - 2x and (x+1)^2 - x^2 = 2x + 1,
    #   so sum d = 2, sum d^2 = 8x^2 + 2.  With Jc = K + x^2:
    #   G2 = (8x^2 + 2)/Jc^2, L = 2/Jc, num = 0.5 G2 - L^2/16 = (4x^2 + 3/4)/Jc^2,
    #   den = 1 + L/4 = 1 + 1/(2 Jc), qsqr = num/den^2.
    K, n, q0 = 40.0, 24, 0.003
    x = np.arange(n, dtype=np.float64)
    prof = K + x ** 2
    J = np.tile(prof, (5, 1)) if axis == 1 else np.tile(prof[:, None], (1, 5))
    c = oracle.srad_coeff(J, q0)
    line = c[2, :] if axis == 1 else c[:, 2]
    for xi in range(1, n - 1):
        jc = K + xi ** 2
        q = ((4 * xi ** 2 + 0.75) / jc ** 2) / (1 + 0.5 / jc) ** 2
        assert line[xi] == pytest.approx(_c_from_q(q, q0), rel=1e-12), xi
    # the profile spans both clamp branches (c = 1 where qsqr < q0, c < 1 elsewhere)
    assert line.max() == 1.0 and line.min() < 0.5


def test_linear_ramp_coefficient():
    # J = K + b x: differences -b, +b => L = 0, G2 = 2 b^2/Jc^2, qsqr = b^2/Jc^2.
    K, b, q0 = 10.0, 0.3, 1e-4
    J = np.tile(K + b * np.arange(16.0), (3, 1))
    c = oracle.srad_coeff(J, q0)
    for xi in range(1, 15):
        jc = K + b * xi
        assert c[1, xi] == pytest.approx(_c_from_q(b * b / jc ** 2, q0), rel=1e-13)


@pytest.mark.parametrize("R,C,m,q", [(20, 28, 2, 3), (9, 16, 5, 1)])
def test_saturated_coefficient_is_5pt_diffusion_eigenmode(R, C, m, q):
    # With q0sqr far above every qsqr, t < 0 => c > 1 => clamped to 1, and one iteration is
    # J' = J + (lambda/4) (dN + dS + dW + dE): the clamped 5-point diffusion, whose cosine
    # modes decay by g = 1 - lambda (sin^2(pi m/2C) + sin^2(pi q/2R)) per iteration.
    lam, n, M, eps = 0.5, 12, 3.0, 0.01
    jj = (np.arange(C) + 0.5) / C
    ii = (np.arange(R) + 0.5) / R
    mode = np.outer(np.cos(np.pi * q * ii), np.cos(np.pi * m * jj))
    J = M + eps * mode
    assert np.all(oracle.srad_coeff(J, 1e6) == 1.0)
    for _ in range(n):
        J = oracle.srad_step(J, 1e6, lam)
    g = 1 - lam * (np.sin(np.pi * m / (2 * C)) ** 2 + np.sin(np.pi * q / (2 * R)) ** 2)
    np.testing.assert_allclose(J - M, g ** n * eps * mode, rtol=0, atol=1e-14)


def test_uniform_image_unchanged_bit_exact():
    J = np.full((12, 15), 2.0)
    assert np.array_equal(oracle.srad(J, 0, 5, 0, 5, 0.5, 20), J)
    assert np.all(oracle.srad_coeff(J, 0.0) == 1.0)


def test_lambda_zero_unchanged():
    rng = np.random.default_rng(3)
    J = np.exp(rng.random((14, 11)))
    assert np.array_equal(oracle.srad(J, 0, 6, 0, 6, 0.0, 5), J)


def test_exact_one_iteration_footprint():
    # new J(i,j) reads old J at (i,j), (i+-1,j), (i,j+-1) [differences and c(i,j)],
    # (i+2,j), (i+1,j+-1) [through c(i+1,j)], (i,j+2), (i-1,j+1) [through c(i,j+1)].
    # So a perturbation at (r,c) changes exactly the cells (r-di, c-dj) for
    # (di,dj) in F = {(0,0),(+-1,0),(0,+-1),(2,0),(1,+-1),(0,2),(-1,1)}.
    # The ROI is nearly flat (q0 ~ 1e-8) so c is far from its clamps near the noisy spot.
    rng = np.random.default_rng(4)
    R, C, r, c = 24, 24, 12, 11
    J = np.exp(rng.random((R, C)))
    J[:6, :6] = 2.0 + 1e-4 * rng.random((6, 6))
    q0 = oracle.srad_q0sqr(J, 0, 5, 0, 5)
    base = oracle.srad_step(J, q0, 0.5)
    Jp = J.copy()
    Jp[r, c] += 0.05
    pert = oracle.srad_step(Jp, q0, 0.5)
    changed = {tuple(x) for x in np.argwhere(pert != base)}
    F = {(0, 0), (1, 0), (-1, 0), (0, 1), (0, -1), (2, 0), (1, 1), (1, -1), (0, 2), (-1, 1)}
    assert changed == {(r - di, c - dj) for di, dj in F}


def test_max_principle():
    rng = np.random.default_rng(5)
    J0 = np.exp(rng.random((30, 30)))
    for lam in (0.5, 1.0):
        J = oracle.srad(J0, 0, 9, 0, 9, lam, 25)
        assert J.min() >= J0.min() - 1e-12 and J.max() <= J0.max() + 1e-12


def test_dependency_cone_outside_unchanged():
    # Noisy ROI block on a constant background: after t iterations a cell can only have been
    # influenced from rows [i - t, i + 2t] ... equivalently the perturbation spreads at most
    # 2 rows/cols toward lower indices and 1 toward higher ones per iteration.
    rng = np.random.default_rng(6)
    R = C = 40
    J = np.full((R, C), 1.5)
    r1, r2, c1, c2 = 15, 22, 16, 24
    J[r1:r2 + 1, c1:c2 + 1] = np.exp(rng.random((r2 - r1 + 1, c2 - c1 + 1)))
    t = 4
    out = oracle.srad(J, r1, r2, c1, c2, 0.5, t)
    mask = np.zeros((R, C), bool)
    mask[max(r1 - 2 * t, 0):r2 + t + 1, max(c1 - 2 * t, 0):c2 + t + 1] = True
    assert np.array_equal(out[~mask], J[~mask])
    assert not np.array_equal(out[mask], J[mask])


# ----------------------------------------------------------------------------- srad_v1
def test_srad_v1_is_extract_v2_whole_roi_compress():
    # Rodinia srad_v1 = extract (exp(x/255)) + srad_v2 iterations with ROI = whole image +
    # compress (log(J)*255) -- composition of independently pinned pieces
    import synth
    img = synth.srad_v1_image(37, 29)
    J = np.exp(img.astype(np.float64) / 255.0)
    ref = np.log(oracle.srad(J, 0, 36, 0, 28, 0.5, 6)) * 255.0
    np.testing.assert_allclose(oracle.srad_v1(img, 0.5, 6), ref, rtol=0, atol=1e-10)


def test_srad_v1_fixed_points():
    import synth
    img = synth.srad_v1_image(30, 40)
    # lambda = 0 and niter = 0: only the exp/log round trip
    np.testing.assert_allclose(oracle.srad_v1(img, 0.0, 5), img, rtol=0, atol=1e-9)
    np.testing.assert_allclose(oracle.srad_v1(img, 0.5, 0), img, rtol=0, atol=1e-9)
    flat = np.full((16, 20), 97.0)
    np.testing.assert_allclose(oracle.srad_v1(flat, 0.5, 10), flat, rtol=0, atol=1e-9)


def test_srad_v1_smooths_speckle():
    # anisotropic diffusion reduces the coefficient of variation of a speckled image
    import synth
    img = synth.srad_v1_image(64, 64)
    out = oracle.srad_v1(img, 0.5, 30)
    def cv(a):
        J = np.exp(a / 255.0)
        return J.std() / J.mean()
    assert cv(out) < 0.8 * cv(img)
    assert out.min() >= img.min() - 1e-9 and out.max() <= img.max() + 1e-9  # maximum principle
