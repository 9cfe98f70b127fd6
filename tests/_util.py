"""Test helpers: windowed oracle evaluation for sampled outputs at full problem sizes.

A stencil output cell after n steps depends only on its dependency cone.  Evaluating the
plain oracle on a window around the cell that extends the cone by a safety margin gives
the exact value: wrong values generated at the window's artificial edges travel at most one
cell per step and never reach the centre.  Where the window touches the real grid edge it
coincides with it, so the clamp boundary is reproduced exactly.
"""
from __future__ import annotations

import numpy as np

import oracle


def hotspot_window_value(T, P, i, j, iters, coef):
    """Oracle value of hotspot cell (i, j) after `iters` steps (fp64), via a window."""
    R, C = T.shape
    r = iters + 1
    i0, i1 = max(0, i - r), min(R, i + r + 1)
    j0, j1 = max(0, j - r), min(C, j + r + 1)
    out = oracle.hotspot(T[i0:i1, j0:j1], P[i0:i1, j0:j1], iters, coef["k"], coef["rx"],
                         coef["ry"], coef["rz"], coef["amb"])
    return out[i - i0, j - j0]


def srad_window_value(J, i, j, niter, q0_seq, lam):
    """Oracle value of srad cell (i, j) after niter iterations given the q0sqr sequence of the
    full grid.  One iteration reads rows i-1..i+2 / cols j-1..j+2, so the cone after n
    iterations spans rows [i-n, i+2n], cols [j-n, j+2n]; the window adds a margin of 2n."""
    R, C = J.shape
    m = 2 * niter + 2
    i0, i1 = max(0, i - m), min(R, i + m + 1)
    j0, j1 = max(0, j - m), min(C, j + m + 1)
    w = np.asarray(J[i0:i1, j0:j1], dtype=np.float64)
    for t in range(niter):
        w = oracle.srad_step(w, q0_seq[t], lam)
    return w[i - i0, j - j0]


def rel_err(a, b):
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    return np.max(np.abs(a - b) / np.maximum(np.abs(b), 1e-30)) if a.size else 0.0


def hotspot_window_block(T, P, i0, j0, h, w, iters, coef):
    """Oracle values (fp64) of the h x w output block at (i0, j0) after `iters` steps: the plain
    oracle on the block grown by the cone radius iters + 1 (clamped to the grid, where the
    window then coincides with the real boundary)."""
    R, C = T.shape
    r = iters + 1
    a0, a1 = max(0, i0 - r), min(R, i0 + h + r)
    b0, b1 = max(0, j0 - r), min(C, j0 + w + r)
    out = oracle.hotspot(T[a0:a1, b0:b1], P[a0:a1, b0:b1], iters, coef["k"], coef["rx"],
                         coef["ry"], coef["rz"], coef["amb"])
    return out[i0 - a0:i0 - a0 + h, j0 - b0:j0 - b0 + w]


def srad_window_block(J, i0, j0, h, w, niter, q0_seq, lam):
    """Oracle values of the h x w srad output block at (i0, j0) after niter iterations, given the
    full grid's q0sqr sequence; window = block grown by 2*niter + 2 on every side (the cone
    reaches niter rows/cols toward lower and 2*niter toward higher indices)."""
    R, C = J.shape
    m = 2 * niter + 2
    a0, a1 = max(0, i0 - m), min(R, i0 + h + m)
    b0, b1 = max(0, j0 - m), min(C, j0 + w + m)
    x = np.asarray(J[a0:a1, b0:b1], dtype=np.float64)
    for t in range(niter):
        x = oracle.srad_step(x, q0_seq[t], lam)
    return x[i0 - a0:i0 - a0 + h, j0 - b0:j0 - b0 + w]
