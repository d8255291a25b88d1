"""Pins of oracle O0-O2 (SpMM Alg 1, SDDMM Alg 2) against things other
than the oracle: dense brute force through numpy matmul, SpMV at K=1, bitwise row-
permutation equivariance, pattern preservation.  CPU only."""
import numpy as np
import pytest

from synth import generators as g


def dense_of(A):
    D = np.zeros((A.nrows, A.ncols), np.float64)
    r = np.repeat(np.arange(A.nrows), np.diff(A.rowptr))
    D[r, A.colidx] = A.vals
    return D


CASES = [
    (17, 23, 0.2, 0.0, 1),
    (64, 64, 0.1, 0.3, 2),   # ~30% empty rows
    (40, 7, 0.5, 0.1, 3),    # M != N, dense-ish
    (1, 50, 0.3, 0.0, 4),    # single row
    (33, 1, 0.6, 0.0, 5),    # single column
]


@pytest.mark.parametrize("M,N,dens,empty,seed", CASES)
@pytest.mark.parametrize("K", [1, 3, 16])
def test_spmm_matches_dense_bruteforce(oracle, M, N, dens, empty, seed, K):
    A = g.random_csr(M, N, dens, seed, empty_frac=empty)
    B = g.dense(N, K, seed=seed)
    ref = dense_of(A) @ B.astype(np.float64)
    got = oracle.spmm(A, B)
    np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("M,N,dens,empty,seed", CASES)
@pytest.mark.parametrize("K", [1, 5, 16])
def test_sddmm_matches_dense_bruteforce(oracle, M, N, dens, empty, seed, K):
    A = g.random_csr(M, N, dens, seed, empty_frac=empty)
    X = g.dense(M, K, seed=seed, stream=1)
    Y = g.dense(N, K, seed=seed, stream=2)
    full = (X.astype(np.float64) @ Y.astype(np.float64).T) * dense_of(A)
    r = np.repeat(np.arange(A.nrows), np.diff(A.rowptr))
    got, gabs = oracle.sddmm(A, X, Y)
    np.testing.assert_allclose(got, full[r, A.colidx], rtol=1e-12, atol=1e-12)
    # bound scale |a|·Σ|x||y| dominates |out|
    assert np.all(np.abs(got) <= gabs * (1 + 1e-12))


def test_sddmm_output_keeps_pattern(oracle):
    """O has S's pattern: scattering out into an MxN matrix has support ⊆ S."""
    A = g.random_csr(30, 30, 0.15, 9, empty_frac=0.2)
    X, Y = g.dense(30, 8, stream=1), g.dense(30, 8, stream=2)
    out, _ = oracle.sddmm(A, X, Y)
    O = np.zeros((30, 30))
    r = np.repeat(np.arange(30), np.diff(A.rowptr))
    O[r, A.colidx] = out
    assert np.all((O != 0) <= (dense_of(A) != 0))
    assert out.shape == (A.nnz,)


def test_spmv_special_case(oracle):
    """K = 1 reduces Alg 1 to SpMV."""
    A = g.random_csr(50, 40, 0.2, 12)
    x = g.dense(40, 1)
    np.testing.assert_allclose(oracle.spmm(A, x)[:, 0], dense_of(A) @ x[:, 0].astype(np.float64),
                               rtol=1e-13, atol=1e-13)


def test_row_permutation_equivariance_bitwise(oracle):
    """oracle(P·A) = P·oracle(A) bitwise: each row's nnz order is unchanged."""
    A = g.random_csr(64, 48, 0.2, 21, empty_frac=0.2)
    B = g.dense(48, 12)
    perm = np.random.default_rng(5).permutation(64)
    deg = np.diff(A.rowptr)
    rp = np.zeros(65, np.int64)
    np.cumsum(deg[perm], out=rp[1:])
    ci = np.concatenate([A.colidx[A.rowptr[r]:A.rowptr[r + 1]] for r in perm])
    vv = np.concatenate([A.vals[A.rowptr[r]:A.rowptr[r + 1]] for r in perm])
    PA = g.CSR(64, 48, rp, ci.astype(np.int32), vv.astype(np.float32))
    assert np.array_equal(oracle.spmm(PA, B), oracle.spmm(A, B)[perm])
    X, Y = g.dense(64, 12, stream=1), g.dense(48, 12, stream=2)
    o1, _ = oracle.sddmm(PA, X[perm], Y)
    o0, _ = oracle.sddmm(A, X, Y)
    o0p = np.concatenate([o0[A.rowptr[r]:A.rowptr[r + 1]] for r in perm])
    assert np.array_equal(o1, o0p)


def test_spmm_rows_matches_full(oracle):
    A = g.random_csr(80, 60, 0.1, 31, empty_frac=0.1)
    B = g.dense(60, 9)
    rows = np.array([0, 5, 79, 41, 5])
    c, cabs = oracle.spmm_rows(A, B, rows)
    np.testing.assert_array_equal(c, oracle.spmm(A, B)[rows])
    bound = np.abs(dense_of(A)) @ np.abs(B.astype(np.float64))
    np.testing.assert_allclose(cabs, bound[rows], rtol=1e-12)


def test_canonicalize_sorts_and_tracks_positions(oracle):
    A = g.random_csr(40, 40, 0.2, 3)
    U = g.shuffle_within_rows(A, seed=4)
    assert not np.array_equal(U.colidx, A.colidx)
    col, val, pos = oracle.canonicalize(U)
    np.testing.assert_array_equal(col, A.colidx)
    np.testing.assert_array_equal(val, A.vals)
    np.testing.assert_array_equal(U.colidx[pos], col)
    # Alg 1 is order-insensitive up to rounding
    np.testing.assert_allclose(oracle.spmm(U, g.dense(40, 4)), oracle.spmm(A, g.dense(40, 4)), rtol=1e-12)


def test_canonicalize_rejects_bad_input(oracle):
    A = g.fig1a()
    dup = g.CSR(6, 6, A.rowptr, A.colidx.copy(), A.vals)
    dup.colidx[1] = 0  # row 0 = {0, 0}
    with pytest.raises(ValueError):
        oracle.canonicalize(dup)
    oob = g.CSR(6, 6, A.rowptr, A.colidx.copy(), A.vals)
    oob.colidx[3] = 6
    with pytest.raises(ValueError):
        oracle.canonicalize(oob)
    bad = g.CSR(6, 6, A.rowptr.copy(), A.colidx, A.vals)
    bad.rowptr[2] = 1  # decreasing
    with pytest.raises(ValueError):
        oracle.canonicalize(bad)


@pytest.mark.parametrize("M,N,dens,empty,seed", CASES)
@pytest.mark.parametrize("K", [1, 7, 16])
def test_sddmm_bound_scale_elementwise(oracle, M, N, dens, empty, seed, K):
    """The tolerance scale of every GPU SDDMM check (north_star: |err| <= 1e-4·Σ|a||x||y|)
    is out_abs[p] = |a_ij|·Σ_k |x_ik|·|y_jk|: pinned element by element against numpy's
    (|X| @ |Y|ᵀ) ⊙ |A| in fp64, not only as an upper bound of |out|."""
    A = g.random_csr(M, N, dens, seed, empty_frac=empty)
    X = g.dense(M, K, seed=seed, stream=1)
    Y = g.dense(N, K, seed=seed, stream=2)
    full = (np.abs(X.astype(np.float64)) @ np.abs(Y.astype(np.float64)).T) * np.abs(dense_of(A))
    r = np.repeat(np.arange(A.nrows), np.diff(A.rowptr))
    _, gabs = oracle.sddmm(A, X, Y)
    np.testing.assert_allclose(gabs, full[r, A.colidx], rtol=1e-12, atol=0)
