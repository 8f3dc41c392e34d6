"""Invariants of the seeded input generator (xgcgen): shape, determinism,
partition independence, strict diagonal dominance, species calibration
(Fig. 2; Table III, calibration only)."""
import numpy as np
import scipy.sparse as sp

import xgcgen as X


def test_pattern_shape_and_sorted():
    pat = X.stencil_pattern()
    assert pat.n == 992 and pat.nnz == 8554 and pat.max_row_nnz == 9
    for i in range(pat.n):
        cols = pat.col_idx[pat.row_ptr[i]:pat.row_ptr[i + 1]]
        assert np.all(np.diff(cols) > 0) and i in cols


def test_transposed_grid():
    pat = X.stencil_pattern(31, 32)
    assert pat.n == 992 and pat.nnz == 8554


def test_determinism_and_partition_independence():
    a = X.make_batch(0, 40, chunk=7, threads=3)
    b = X.make_batch(17, 13, chunk=5, threads=1)
    assert np.array_equal(a.values[17:30], b.values) and np.array_equal(a.b[17:30], b.b)
    c = X.make_batch(0, 40, seed=X.DEFAULT_SEED + 1)
    assert not np.array_equal(a.values, c.values)


def test_strict_diagonal_dominance_and_nonsymmetry():
    B = X.make_batch(0, 6)
    pat = B.pattern
    for k in range(6):
        A = sp.csr_matrix((B.values[k], pat.col_idx, pat.row_ptr), shape=(pat.n, pat.n))
        d = np.abs(A.diagonal())
        off = np.abs(A).sum(axis=1).A1 - d
        assert np.all(d - off >= 1.0 - 1e-12)        # margin = 1
        assert abs(A - A.T).max() > 0                  # not symmetric


def test_species_eigenvalues_fig2():
    """Ion eigenvalues cluster near 1, electron real parts spread wider (Fig. 2)."""
    B = X.make_batch(0, 2)
    pat = B.pattern
    ev = []
    for k in range(2):
        A = sp.csr_matrix((B.values[k], pat.col_idx, pat.row_ptr), shape=(pat.n, pat.n)).toarray()
        ev.append(np.linalg.eigvals(A).real)
    ion, ele = ev
    assert ion.min() > 0.9 and ion.max() < 2.0
    assert ele.max() / ele.min() > 5.0


def test_ell_conversion_roundtrip():
    B = X.make_batch(0, 3)
    pat = B.pattern
    ell = X.csr_values_to_ell(B.values, pat.row_ptr, pat.col_idx)
    ell_col, src = X.ell_layout(pat.row_ptr, pat.col_idx)
    assert ell.shape == (3, 9 * pat.n)
    assert np.all(ell[:, src < 0] == 0.0)
    n = pat.n
    for e in (0, 100, 5000, pat.nnz - 1):
        i = int(np.searchsorted(pat.row_ptr, e, side="right") - 1)
        k = e - pat.row_ptr[i]
        assert ell_col[k * n + i] == pat.col_idx[e]
        assert np.array_equal(ell[:, k * n + i], B.values[:, e])
