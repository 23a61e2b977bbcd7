"""Generator sanity (lfgen): shapes of BASELINE.json configs, symmetry, Table 3 sizes."""
import numpy as np

import lfgen


def _symmetric(A):
    rows = np.repeat(np.arange(A.N, dtype=np.int64), np.diff(A.rowptr))
    k1 = rows * A.N + A.col
    k2 = A.col.astype(np.int64) * A.N + rows
    o1, o2 = np.argsort(k1), np.argsort(k2)
    return np.array_equal(k1[o1], k2[o2]) and np.array_equal(A.val[o1], A.val[o2])


def test_c1_shape():
    A = lfgen.config("C1")
    assert A.N == 4096 and A.nnz == 20224 and A.n_edges == 8064
    assert _symmetric(A)


def test_aniso_table3_sizes():
    """ANISO1/2 at 2500^2: N = 6,250,000 and nnz = 56,220,004 (Table 3)."""
    for kind in (1, 2):
        A = lfgen.aniso2d(2500, kind)
        assert A.N == 6_250_000 and A.nnz == 56_220_004


def test_small_replicas_symmetric_and_sorted():
    for A in (lfgen.grid3d_7pt_aniso(10), lfgen.fem27_bricks(10), lfgen.chung_lu(2000),
              lfgen.grid3d_27pt(8), lfgen.random_graph(50, 100, seed=1, ties=True)):
        assert _symmetric(A), A.name
        assert A.rowptr[0] == 0 and np.all(np.diff(A.rowptr) >= 0)
        for v in range(0, A.N, max(1, A.N // 50)):
            c = A.col[A.rowptr[v]:A.rowptr[v + 1]]
            assert np.all(np.diff(c) > 0)


def test_deterministic():
    a, b = lfgen.fem27_bricks(10), lfgen.fem27_bricks(10)
    assert np.array_equal(a.col, b.col) and np.array_equal(a.val, b.val)
    c = lfgen.grid3d_27pt(8)
    assert c.n_edges == _e27(8)


def _e27(n):
    """Undirected 27-point couplings on n^3: sum over the 13 forward offsets."""
    tot = 0
    for dz in (-1, 0, 1):
        for dy in (-1, 0, 1):
            for dx in (-1, 0, 1):
                if (dz, dy, dx) > (0, 0, 0):
                    tot += (n - abs(dx)) * (n - abs(dy)) * (n - abs(dz))
    return tot


def test_c5_edge_count_formula():
    """C5 512^3 has 1,737,761,788 undirected edges (SURVEY.md §8(a) size table)."""
    assert _e27(512) == 1_737_761_788


def test_slab_rows_equal_global_rows():
    """Per-rank slab generation equals the rows of the whole graph (multi-GPU bench)."""
    n, nz = 10, 12
    A = lfgen.grid3d_7pt_aniso(n)  # nz == n here only for the first check below
    rp, col, val, lo, hi = lfgen.grid3d_7pt_aniso_rows(n, n, 3, 7)
    a, b = A.rowptr[lo], A.rowptr[hi]
    assert np.array_equal(rp, A.rowptr[lo:hi + 1] - a)
    assert np.array_equal(col, A.col[a:b]) and np.array_equal(val.view(np.uint32), A.val[a:b].view(np.uint32))
    # a taller grid: rows of consecutive slabs concatenate to the full matrix
    parts = [lfgen.grid3d_7pt_aniso_rows(n, nz, z0, z1) for z0, z1 in ((0, 5), (5, 12))]
    assert parts[0][4] == parts[1][3] and parts[1][4] == n * n * nz
