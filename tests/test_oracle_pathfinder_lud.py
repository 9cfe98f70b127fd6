"""Pins for the pathfinder and lud oracles (CPU only).

pathfinder: brute-force path enumeration on tiny grids, constant walls, single column,
single row, the row-minimum lower bound.
lud: the Kac-Murdock-Szego closed-form factors of Rodinia's matrix, exact recovery of
integer factors, scipy's partial-pivoting LU on column-diagonally-dominant matrices (where
no pivot is ever taken), numpy's Cholesky for SPD matrices, triangular/identity cases.
"""
import itertools

import numpy as np
import pytest
import scipy.linalg

import oracle
import synth


# ----------------------------------------------------------------------------- pathfinder
def _brute_force(wall):
    R, C = wall.shape
    best = np.full(C, np.iinfo(np.int64).max, dtype=np.int64)
    for start in range(C):
        for moves in itertools.product((-1, 0, 1), repeat=R - 1):
            j, cost, ok = start, int(wall[0, start]), True
            for r, mv in enumerate(moves, start=1):
                j += mv
                if not 0 <= j < C:
                    ok = False
                    break
                cost += int(wall[r, j])
            if ok:
                best[j] = min(best[j], cost)
    return best


def test_pathfinder_brute_force_tiny_grids():
    rng = np.random.default_rng(11)
    for _ in range(120):
        R, C = rng.integers(1, 7), rng.integers(1, 8)
        wall = rng.integers(0, 10, size=(R, C)).astype(np.int32)
        assert np.array_equal(oracle.pathfinder(wall), _brute_force(wall)), (R, C)


def test_pathfinder_constant_wall():
    assert np.all(oracle.pathfinder(np.full((100, 37), 7, np.int32)) == 700)


def test_pathfinder_single_column_and_row():
    w = synth.pathfinder_wall(50, 1)
    assert oracle.pathfinder(w)[0] == w.sum()
    w = synth.pathfinder_wall(1, 40)
    assert np.array_equal(oracle.pathfinder(w), w[0])


def test_pathfinder_lower_bound_and_values():
    w = synth.pathfinder_wall(30, 200)
    res = oracle.pathfinder(w)
    assert np.all(res >= w.min(axis=1).sum())
    assert np.all(res <= w[:, :].max(axis=1).sum())


# ----------------------------------------------------------------------------- lud
def test_lud_kms_closed_form():
    # A = 10 * KMS(rho), rho = e^-0.001 (Rodinia create_matrix, fp64).  KMS = L D L^T with
    # L[i][j] = rho^(i-j) and D = diag(1, 1-rho^2, ...), so Doolittle gives
    # L[i][j] = rho^(i-j), U[0][j] = 10 rho^j, U[i][j] = 10 (1-rho^2) rho^(j-i) (i >= 1).
    n = 300
    rho = np.exp(-0.001)
    i = np.arange(n, dtype=np.float64)
    A = 10.0 * np.exp(-0.001 * np.abs(i[:, None] - i[None, :]))
    L, U = oracle.lud_unpack(oracle.lud(A))
    d = i[:, None] - i[None, :]
    L_ref = np.where(d >= 0, rho ** np.maximum(d, 0), 0.0)
    U_ref = np.where(d <= 0, 10 * (1 - rho ** 2) * rho ** np.maximum(-d, 0), 0.0)
    U_ref[0, :] = 10 * rho ** i
    np.testing.assert_allclose(L, L_ref, rtol=1e-9, atol=1e-12)
    np.testing.assert_allclose(U, U_ref, rtol=1e-9, atol=1e-12)


@pytest.mark.parametrize("n", [1, 7, 64, 200])
def test_lud_integer_factors_exact(n):
    A, L0, U0 = synth.lud_integer_factors(n)
    L, U = oracle.lud_unpack(oracle.lud(A))
    assert np.array_equal(L, L0) and np.array_equal(U, U0)


@pytest.mark.parametrize("n", [5, 50, 160])
def test_lud_matches_scipy_no_pivot_case(n):
    # A^T strictly diagonally dominant by columns => partial pivoting never swaps rows.
    A = synth.lud_diag_dominant(n).astype(np.float64)
    P, Ls, Us = scipy.linalg.lu(A)
    assert np.array_equal(P, np.eye(n))
    L, U = oracle.lud_unpack(oracle.lud(A))
    np.testing.assert_allclose(L, Ls, rtol=1e-12, atol=1e-14)
    np.testing.assert_allclose(U, Us, rtol=1e-12, atol=1e-12)


def test_lud_cholesky_relation():
    rng = np.random.default_rng(8)
    B = rng.random((40, 40))
    A = B @ B.T + 40 * np.eye(40)
    L, U = oracle.lud_unpack(oracle.lud(A))
    G = np.linalg.cholesky(A)
    np.testing.assert_allclose(G, L * np.sqrt(np.diag(U))[None, :], rtol=1e-11, atol=1e-12)


def test_lud_triangular_and_identity():
    rng = np.random.default_rng(9)
    Uonly = np.triu(rng.random((12, 12))) + np.eye(12)
    L, U = oracle.lud_unpack(oracle.lud(Uonly))
    assert np.array_equal(L, np.eye(12)) and np.array_equal(U, Uonly)
    assert np.array_equal(oracle.lud(np.eye(9)), np.eye(9))


def test_lud_backward_error_rodinia_matrix():
    A = synth.lud_rodinia_matrix(256).astype(np.float64)
    L, U = oracle.lud_unpack(oracle.lud(A))
    assert np.abs(L @ U - A).max() / np.abs(A).max() < 1e-13
