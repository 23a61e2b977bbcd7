"""Pins of the oracle's general-input path (§4, §5.1):
S = A' + A'^T and "pi from the underlying undirected graph, coefficients from the original
graph".  Each pin is independent of the oracle's own code path:
  - symmetric input: S is exactly 2|A| off the diagonal, and the whole general pipeline
    reduces to the symmetric one (a positive scale keeps every key order and tie);
  - dense brute force: |A| + |A|^T with the diagonal removed, as a dense float32 sum;
  - the tridiagonal of Q^T A Q on the forest edges, from the dense non-symmetric A.
"""
import numpy as np
import pytest

import lfgen
import oracle


def _dense_pattern(A):
    P = np.zeros((A.N, A.N), dtype=bool)
    rows = np.repeat(np.arange(A.N), np.diff(A.rowptr))
    P[rows, A.col] = True
    return P


def _dense32(A):
    D = np.zeros((A.N, A.N), dtype=np.float32)
    rows = np.repeat(np.arange(A.N), np.diff(A.rowptr))
    D[rows, A.col] = A.val
    return D


@pytest.mark.parametrize("base", ["c1", "rand"])
def test_symmetric_input_reduces_to_symmetric_pipeline(base):
    A = lfgen.grid2d_5pt(16, seed=1) if base == "c1" else lfgen.random_graph(300, 900, seed=5, ties=True)
    S = oracle.symmetrize(A)
    rows = np.repeat(np.arange(A.N), np.diff(A.rowptr))
    off = rows != A.col
    assert np.array_equal(S.rowptr, np.concatenate([[0], np.cumsum(np.bincount(rows[off], minlength=A.N))]))
    assert np.array_equal(S.col, A.col[off])
    assert np.array_equal(S.val, (np.float32(2) * np.abs(A.val[off])).astype(np.float32))
    g = oracle.run_pipeline_general(A)
    o = oracle.run_pipeline(A)
    for k in ("pi", "forest", "path_id", "pos", "perm", "iperm"):
        assert np.array_equal(g[k], o[k]), k
    for k in ("a", "b", "c"):
        assert np.array_equal(g[k].view(np.uint32), o[k].view(np.uint32)), k
    assert np.array_equal(g["pi_w"], np.float32(2) * o["pi_w"])


@pytest.mark.parametrize("seed", [1, 2, 3])
@pytest.mark.parametrize("ties", [False, True])
def test_symmetrize_dense_brute_force(seed, ties):
    A = lfgen.nonsymmetric(lfgen.random_graph(40, 120, seed=seed), seed=seed, drop=0.3, zeros=0.1, ties=ties)
    S = oracle.symmetrize(A)
    D = np.abs(_dense32(A))
    want = (D + D.T).astype(np.float32)
    np.fill_diagonal(want, 0)
    P = _dense_pattern(A)
    pat = P | P.T
    np.fill_diagonal(pat, False)
    assert np.array_equal(_dense_pattern(S), pat)
    assert np.array_equal(_dense32(S), want)
    for i in range(S.N):  # rows ascending
        c = S.col[S.rowptr[i]:S.rowptr[i + 1]]
        assert np.all(np.diff(c) > 0)


@pytest.mark.parametrize("seed", [4, 5])
def test_general_tridiag_is_QtAQ_on_forest_edges(seed):
    A = lfgen.nonsymmetric(lfgen.grid2d_5pt(10, seed=seed), seed=seed, drop=0.25, zeros=0.05)
    g = oracle.run_pipeline_general(A)
    perm = g["perm"]
    T = _dense32(A)[np.ix_(perm, perm)]  # (Q^T A Q)_{rs} = a_{perm[r], perm[s]}
    f = g["forest"].reshape(-1, 2)
    N = A.N
    for r in range(N):
        v = perm[r]
        assert g["b"][r] == T[r, r]
        exp_a = T[r, r - 1] if r > 0 and perm[r - 1] in f[v] else np.float32(0)
        exp_c = T[r, r + 1] if r + 1 < N and perm[r + 1] in f[v] else np.float32(0)
        assert g["a"][r] == exp_a and g["c"][r] == exp_c, r


def test_general_factor_is_a_factor_of_S():
    A = lfgen.nonsymmetric(lfgen.grid3d_27pt(8, seed=5), seed=9)
    g = oracle.run_pipeline_general(A)
    S = g["S"]
    P = _dense_pattern(S)
    pi = g["pi"]
    for v in range(A.N):
        for w in pi[v]:
            if w >= 0:
                assert P[v, w] and v in pi[w]
