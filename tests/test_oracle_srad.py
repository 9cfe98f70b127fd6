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


# ----------------------------------------------------------------------------- q0sqr per iteration
def _row_mode(R, C, eps):
    # J = 1 + eps*cos(pi*(i+1/2)/R): the slowest eigenmode of the clamped (Neumann) 5-point
    # Laplacian along rows, constant along columns; eigenvalue -4 sin^2(pi/(2R))
    i = np.arange(R, dtype=np.float64)[:, None]
    return np.repeat(1.0 + eps * np.cos(np.pi * (i + 0.5) / R), C, axis=1)


def test_q0sqr_is_reevaluated_every_iteration_closed_form():
    # Rodinia srad_v2's host loop recomputes the ROI statistics at the top of EVERY iteration
    # (DESIGN.md §3 S1/S2; SURVEY §8(c) srad definition "for it in 0..niter-1: ... s = sum_ROI J").
    # On the row eigenmode with the ROI = whole grid, c saturates at 1 (qsqr ~ (eps*pi/R)^2 is
    # far below q0sqr ~ eps^2/2), so J_t = 1 + eps g^t cos(.) with g = 1 - lambda sin^2(pi/2R):
    # mean_t = 1 (sum of cos over the period is 0), var_t = eps^2 g^(2t) / 2, hence
    #   q0sqr(t) = eps^2 g^(2t) / 2       (closed form, t = 0..niter-1).
    # A "q0sqr computed once" oracle reports eps^2/2 at every t and fails from t = 1.
    R, C, eps, lam, n = 64, 6, 0.25, 0.5, 6
    J = _row_mode(R, C, eps)
    out, q0 = oracle.srad(J, 0, R - 1, 0, C - 1, lam, n, return_q0=True)
    g = 1.0 - lam * np.sin(np.pi / (2 * R)) ** 2
    want = eps ** 2 * g ** (2 * np.arange(n)) / 2.0
    np.testing.assert_allclose(q0, want, rtol=1e-10, atol=0)
    assert q0[1] < q0[0] * (1 - 1e-4)  # the sequence really moves
    np.testing.assert_allclose(out, 1.0 + (J - 1.0) * g ** n, rtol=0, atol=1e-13)


def test_q0sqr_sequence_drives_later_iterations():
    # composition with the independently pinned pieces: iteration t uses q0sqr of J_t (not of
    # J_0).  Random data, ROI in a corner, so c is not saturated and q0 matters for J itself.
    rng = np.random.default_rng(11)
    J0 = np.exp(rng.random((24, 31)))
    r1, r2, c1, c2, lam = 2, 9, 3, 12, 0.5
    J = J0.copy()
    seq = []
    for _ in range(3):
        q = oracle.srad_q0sqr(J, r1, r2, c1, c2)
        seq.append(q)
        J = oracle.srad_step(J, q, lam)
    out, q0 = oracle.srad(J0, r1, r2, c1, c2, lam, 3, return_q0=True)
    assert np.array_equal(q0, np.array(seq))
    assert np.array_equal(out, J)
    frozen = J0.copy()
    for _ in range(3):  # the mutation: q0sqr of J_0 reused
        frozen = oracle.srad_step(frozen, seq[0], lam)
    assert np.abs(frozen - out).max() > 1e-6


def test_srad_v1_extract_compress_scale_closed_form():
    # Reading V1 (Rodinia srad_v1 `extract` J = exp(image/255), `compress` image = log(J)*255;
    # the srad the paper evaluates).  Choose the image so that the extracted J is
    # exactly the row eigenmode: image = 255*log(1 + eps cos(.)).  With the whole-image ROI, c
    # saturates (as above) and J_t = 1 + eps g^t cos(.), so the compressed output is
    #   image_t = 255 * log(1 + eps g^t cos(pi (i+1/2)/R)).
    # Any other extract scale s makes J0 = (1 + eps cos)^(255/s), not an eigenmode; any other
    # compress scale s' multiplies the output by s'/255: both fail this closed form.
    R, C, eps, lam, n = 48, 5, 0.3, 0.5, 7
    i = np.arange(R, dtype=np.float64)[:, None]
    mode = np.repeat(np.cos(np.pi * (i + 0.5) / R), C, axis=1)
    img = 255.0 * np.log(1.0 + eps * mode)
    g = 1.0 - lam * np.sin(np.pi / (2 * R)) ** 2
    want = 255.0 * np.log(1.0 + eps * g ** n * mode)
    np.testing.assert_allclose(oracle.srad_v1(img, lam, n), want, rtol=0, atol=1e-10)
    # negative controls: the same pin evaluated with scale 256 or natural-log units fails
    for s in (256.0, 1.0):
        J = np.exp(img / s)
        bad = s * np.log(oracle.srad(J, 0, R - 1, 0, C - 1, lam, n))
        assert np.abs(bad - want).max() > 1e-6
