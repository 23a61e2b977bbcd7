"""Pins of oracle.tri_solve (applying the tridiagonal preconditioner,
PAPER.md §1, §6, ref. [21]) against what mathematics fixes.  No GPU."""
import numpy as np
import pytest


def test_closed_form_1d_laplacian(oracle_mod):
    """T = tridiag(-1, 2, -1) of size n, x = 1: y_i = i (n + 1 - i) / 2 (1-based),
    the discrete Poisson closed form.  A transposed band or a sign slip fails it."""
    for n in (1, 2, 7, 100):
        a = np.full(n, -1.0)
        c = np.full(n, -1.0)
        b = np.full(n, 2.0)
        y = oracle_mod.tri_solve(a, b, c, np.ones(n))
        i = np.arange(1, n + 1)
        np.testing.assert_allclose(y, i * (n + 1 - i) / 2.0, rtol=1e-12)


def test_nonsymmetric_band_orientation(oracle_mod):
    """Non-symmetric 3x3 check against the hand-inverted system: rows
    [2 1 0; 3 4 5; 0 6 7] with y = (1, 2, 3) give x = (4, 26, 33).  a[r] multiplies
    y[r-1], c[r] multiplies y[r+1]; swapping a and c fails."""
    a = np.array([99.0, 3.0, 6.0])   # a[0] ignored
    b = np.array([2.0, 4.0, 7.0])
    c = np.array([1.0, 5.0, 99.0])   # c[N-1] ignored
    y = oracle_mod.tri_solve(a, b, c, np.array([4.0, 26.0, 33.0]))
    np.testing.assert_allclose(y, [1.0, 2.0, 3.0], rtol=1e-12)


def test_dense_brute_force_and_manufactured(oracle_mod):
    """Random (non-dominant, pivoting needed) systems: equal to a dense solve of the
    explicitly assembled matrix, and recovers a manufactured solution."""
    rng = np.random.default_rng(5)
    for n in (3, 17, 64):
        a, b, c = (rng.uniform(-1, 1, n) for _ in range(3))
        b[::3] *= 1e-3   # small pivots force row interchanges
        T = np.diag(b) + np.diag(a[1:], -1) + np.diag(c[:-1], 1)
        yt = rng.standard_normal(n)
        x = T @ yt
        y = oracle_mod.tri_solve(a, b, c, x)
        np.testing.assert_allclose(y, np.linalg.solve(T, x), rtol=1e-8, atol=1e-10)
        np.testing.assert_allclose(y, yt, rtol=1e-7, atol=1e-9)


def test_block_decoupling(oracle_mod):
    """Where a[r] = c[r-1] = 0 the system splits (path boundaries of the linear forest,
    L219): the whole solve equals the pieces solved separately."""
    rng = np.random.default_rng(9)
    n = 40
    a, c = rng.uniform(-1, 1, n), rng.uniform(-1, 1, n)
    b = rng.uniform(2.5, 3.0, n)
    for r in (10, 11, 25):
        a[r] = 0.0
        c[r - 1] = 0.0
    x = rng.standard_normal(n)
    y = oracle_mod.tri_solve(a, b, c, x)
    bounds = [0, 10, 11, 25, n]
    for s, e in zip(bounds[:-1], bounds[1:]):
        ys = oracle_mod.tri_solve(a[s:e], b[s:e], c[s:e], x[s:e])
        np.testing.assert_allclose(y[s:e], ys, rtol=1e-12, atol=1e-14)


def test_matvec_definition(oracle_mod):
    """tri_matvec agrees with the dense assembled matrix (it is the residual checker)."""
    rng = np.random.default_rng(1)
    n = 9
    a, b, c, y = (rng.standard_normal(n) for _ in range(4))
    T = np.diag(b) + np.diag(a[1:], -1) + np.diag(c[:-1], 1)
    np.testing.assert_allclose(oracle_mod.tri_matvec(a, b, c, y), T @ y, rtol=1e-13)
