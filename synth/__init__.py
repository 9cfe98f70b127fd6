"""Seeded synthetic input generators shared by the oracle tests, the GPU tests and bench.py.

This module holds NONE of the method's arithmetic: it only draws the inputs the paper's
workloads consume (Rodinia v3 input recipes).  Both the
oracle (`oracle/`) and the CUDA path (`paper_conf_cgo_ivanovzdem24_b200`) receive the
arrays produced here; neither side imports the other.

All generators use numpy ``Generator(PCG64(seed))`` so a given (shape, seed) is
reproducible on every host.  Seeds follow SURVEY.md §8(d): hotspot T0 seed 1, power
seed 2, srad J0 seed 7, pathfinder wall seed 9, lud random seed 3.
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "hotspot_inputs",
    "srad_input",
    "srad_v1_image",
    "pathfinder_wall",
    "lud_rodinia_matrix",
    "lud_diag_dominant",
    "lud_integer_factors",
]


def _rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def hotspot_inputs(rows: int, cols: int, seed_t: int = 1, seed_p: int = 2):
    """HotSpot grid: temperature T0 = 323.15 + 20*U[0,1) K, power P = 1e-3*U[0,1) W.

    Rodinia feeds floor-plan derived temperature/power files; the synthetic fields have the
    same range (a few hundred kelvin, milliwatt cells) and exercise the same code paths
    (no data-dependent control flow).  Returns float32 C-contiguous arrays (rows, cols).
    """
    t = (323.15 + 20.0 * _rng(seed_t).random((rows, cols))).astype(np.float32)
    p = (1e-3 * _rng(seed_p).random((rows, cols))).astype(np.float32)
    return t, p


def srad_input(rows: int, cols: int, seed: int = 7):
    """srad_v2 image J0 = exp(U[0,1)) in [1, e) (Rodinia srad_v2 draws exp(rand()/RAND_MAX))."""
    return np.exp(_rng(seed).random((rows, cols))).astype(np.float32)


def srad_v1_image(rows: int, cols: int, seed: int = 13):
    """Synthetic ultrasound-like image for srad_v1 (Rodinia reads a 502x458 PGM; no dataset here):
    a smooth intensity field (sum of low-frequency cosines) times Rayleigh speckle, clipped and
    quantised to integer pixel values 0..255, returned as float32 (rows, cols)."""
    rng = _rng(seed)
    y = np.linspace(0.0, 1.0, rows)[:, None]
    x = np.linspace(0.0, 1.0, cols)[None, :]
    base = 0.55 + 0.25 * np.cos(3.1 * x + 0.7) * np.cos(2.3 * y) + 0.15 * np.cos(7.0 * (x + y))
    speckle = rng.rayleigh(scale=0.8, size=(rows, cols))
    img = np.clip(255.0 * base * speckle / 1.25, 0.0, 255.0)
    return np.rint(img).astype(np.float32)


def pathfinder_wall(rows: int, cols: int, seed: int = 9):
    """pathfinder wall: integers uniform in 0..9 (Rodinia: rand() % 10), int32 (rows, cols)."""
    return _rng(seed).integers(0, 10, size=(rows, cols), dtype=np.int64).astype(np.int32)


def lud_rodinia_matrix(n: int):
    """Rodinia lud `create_matrix`: A[i][j] = 10*exp(-0.001*|i-j|), evaluated in fp64 and
    rounded to fp32 once.  (A scaled Kac-Murdock-Szego matrix with rho = exp(-0.001).)"""
    i = np.arange(n, dtype=np.float64)
    a = 10.0 * np.exp(-0.001 * np.abs(i[:, None] - i[None, :]))
    return a.astype(np.float32)


def lud_diag_dominant(n: int, seed: int = 3):
    """Diagonally dominant random matrix U[0,1) + n*I (fp32), safe for LU without pivoting."""
    a = _rng(seed).random((n, n)) + n * np.eye(n)
    return a.astype(np.float32)


def lud_integer_factors(n: int, seed: int = 5, density: float = 0.1):
    """Integer-factor construction.

    L0: unit lower triangular, strictly-lower entries in {-1, 0, 1} (nonzero with
    probability `density`); U0: upper triangular, strictly-upper entries in {-1, 0, 1},
    diagonal entries in {1, 2, 4}.  A = L0 @ U0 is formed in exact int64 arithmetic.
    Returns (A fp32, L0 fp32, U0 fp32).  Every partial sum of any Doolittle ordering is an
    integer of magnitude <= 4n, exactly representable in fp32 while 4n < 2**24, and every
    division is by a power of two, so an fp32 LU of A returns L0, U0 bit-exactly.
    """
    rng = _rng(seed)
    def tri_entries():
        v = rng.choice(np.array([-1, 1], dtype=np.int64), size=(n, n))
        m = rng.random((n, n)) < density
        return v * m
    l0 = np.tril(tri_entries(), -1) + np.eye(n, dtype=np.int64)
    u0 = np.triu(tri_entries(), 1)
    diag = rng.choice(np.array([1, 2, 4], dtype=np.int64), size=n)
    u0 = u0 + np.diag(diag)
    a = l0 @ u0
    return a.astype(np.float32), l0.astype(np.float32), u0.astype(np.float32)
