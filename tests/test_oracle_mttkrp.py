"""Pins of O-MTTKRP (oracle.c) to things other than itself (CPU only).

Each check fails on a plausible oracle mistake: a dropped factor, a wrong
index/mode, a transposed factor, U^(n) leaking in, a wrong sign, a missing abs.
P:N = line N of PAPER.md.
"""
import itertools

import numpy as np
import pytest
import scipy.sparse as sp

import synth_inputs as si


def _dense_random(dims, density, seed):
    rng = np.random.default_rng(seed)
    X = rng.uniform(-1, 1, size=dims) * (rng.random(dims) < density)
    X = X.astype(np.float32)
    inds = np.array(np.nonzero(X), dtype=np.uint32)
    vals = X[tuple(inds)].astype(np.float32)
    return X, inds, vals


def _khatri_rao(A, B):
    """Eq. 4: column r is a_r (x) b_r; B's row index runs fastest (Kolda-Bader, R#3)."""
    I, R = A.shape
    J, _ = B.shape
    return np.einsum("ir,jr->ijr", A, B).reshape(I * J, R)


def _unfold(X, n):
    """Mode-n matricization X_(n): remaining modes in increasing order, earliest fastest."""
    return np.reshape(np.moveaxis(X, n, 0), (X.shape[n], -1), order="F")


@pytest.mark.parametrize("dims", [(5, 4), (4, 3, 5), (3, 4, 2, 3), (2, 3, 2, 3, 2)])
def test_bruteforce_unfolding_times_krp(oracle_mod, dims):
    """Eq. 3 literally: X_(n) (U^(N) (.) ... (.) U^(n+1) (.) U^(n-1) (.) ... (.) U^(1))."""
    R = 5
    X, inds, vals = _dense_random(dims, 0.6, seed=sum(dims))
    U = si.factors(dims, R, seed=len(dims))
    N = len(dims)
    for n in range(N):
        others = [k for k in range(N) if k != n]
        krp = U[others[-1]].astype(np.float64)
        for k in reversed(others[:-1]):
            krp = _khatri_rao(krp, U[k].astype(np.float64))
        expect = _unfold(X.astype(np.float64), n) @ krp
        got, absum = oracle_mod.mttkrp(dims, inds, vals, n, U)
        np.testing.assert_allclose(got, expect, rtol=1e-12, atol=1e-12)
        assert np.all(absum >= np.abs(got) - 1e-12)


def test_rank1_closed_form(oracle_mod):
    """X = a o b o c (exact dyadic values => fp32 products exact):
    M(i, r) = a_i (b^T B(:, r)) (c^T C(:, r)) for mode 0, cyclic for modes 1, 2."""
    rng = np.random.default_rng(3)
    dims = (40, 30, 20)
    vecs = []
    for d in dims:
        v = np.zeros(d)
        sup = rng.choice(d, size=d // 3, replace=False)
        v[sup] = rng.choice([-2.0, -1.0, -0.5, 0.5, 1.0, 2.0, 4.0], size=sup.shape[0])
        vecs.append(v)
    sup = [np.nonzero(v)[0] for v in vecs]
    coords = np.array(list(itertools.product(*sup)), dtype=np.uint32).T
    vals = (vecs[0][coords[0]] * vecs[1][coords[1]] * vecs[2][coords[2]]).astype(np.float32)
    R = 7
    U = si.factors(dims, R, seed=11)
    for n in range(3):
        o = [k for k in range(3) if k != n]
        expect = np.outer(vecs[n], (vecs[o[0]] @ U[o[0]].astype(np.float64))
                          * (vecs[o[1]] @ U[o[1]].astype(np.float64)))
        got, _ = oracle_mod.mttkrp(dims, coords, vals, n, U)
        np.testing.assert_allclose(got, expect, rtol=1e-12, atol=1e-12)


def test_all_ones_factors_give_slice_sums(oracle_mod):
    """U^(k) = 1 => every column of the result is the mode-n slice sum of values."""
    dims = (30, 20, 25, 7)
    inds, vals = si.uniform_coo(dims, 2000, seed=5)
    R = 3
    U = [np.ones((d, R), np.float32) for d in dims]
    for n in range(4):
        slice_sum = np.bincount(inds[n], weights=vals.astype(np.float64), minlength=dims[n])
        got, absum = oracle_mod.mttkrp(dims, inds, vals, n, U)
        for r in range(R):
            np.testing.assert_allclose(got[:, r], slice_sum, rtol=1e-12, atol=1e-12)
            np.testing.assert_allclose(
                absum[:, r],
                np.bincount(inds[n], weights=np.abs(vals.astype(np.float64)), minlength=dims[n]),
                rtol=1e-12, atol=1e-12)


def test_order2_is_spmm(oracle_mod):
    """N = 2: mode 0 is X U^(1) and mode 1 is X^T U^(0) (scipy.sparse)."""
    dims = (50, 60)
    inds, vals = si.uniform_coo(dims, 700, seed=9)
    R = 6
    U = si.factors(dims, R, seed=2)
    X = sp.coo_matrix((vals.astype(np.float64), (inds[0], inds[1])), shape=dims).tocsr()
    got0, _ = oracle_mod.mttkrp(dims, inds, vals, 0, U)
    got1, _ = oracle_mod.mttkrp(dims, inds, vals, 1, U)
    np.testing.assert_allclose(got0, X @ U[1].astype(np.float64), rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(got1, X.T @ U[0].astype(np.float64), rtol=1e-12, atol=1e-12)


def test_rank_one_column_is_chained_ttv(oracle_mod):
    """R = 1: mode-0 MTTKRP = (X x_3 c) x_2 b, two TTVs of Eq. 1."""
    dims = (15, 12, 18)
    inds, vals = si.uniform_coo(dims, 600, seed=4)
    U = si.factors(dims, 1, seed=8)
    b, c = U[1][:, 0].astype(np.float64), U[2][:, 0].astype(np.float64)
    Y = {}
    for x in range(vals.shape[0]):  # TTV along mode 3: y_ij = sum_k x_ijk c_k
        key = (int(inds[0, x]), int(inds[1, x]))
        Y[key] = Y.get(key, 0.0) + float(vals[x]) * c[inds[2, x]]
    z = np.zeros(dims[0])
    for (i, j), y in Y.items():  # TTV along mode 2: z_i = sum_j y_ij b_j
        z[i] += y * b[j]
    got, _ = oracle_mod.mttkrp(dims, inds, vals, 0, U)
    np.testing.assert_allclose(got[:, 0], z, rtol=1e-12, atol=1e-12)


def test_invariants(oracle_mod):
    """Linearity in val and in each U^(k) (k != n); invariance to nonzero order;
    mode-permutation symmetry; U^(n) is never read; abs-sum bounds |result|."""
    dims = (20, 16, 12)
    inds, vals = si.uniform_coo(dims, 900, seed=21)
    R = 4
    U = si.factors(dims, R, seed=3)
    for n in range(3):
        base, absum = oracle_mod.mttkrp(dims, inds, vals, n, U)
        assert np.all(absum + 1e-12 >= np.abs(base))
        two, _ = oracle_mod.mttkrp(dims, inds, (2 * vals).astype(np.float32), n, U)
        np.testing.assert_allclose(two, 2 * base, rtol=1e-12, atol=1e-12)
        neg, _ = oracle_mod.mttkrp(dims, inds, (-vals).astype(np.float32), n, U)
        np.testing.assert_allclose(neg, -base, rtol=1e-12, atol=1e-12)
        for k in range(3):
            if k == n:
                continue
            U2 = list(U)
            U2[k] = (U[k] * 0.5).astype(np.float32)
            half, _ = oracle_mod.mttkrp(dims, inds, vals, n, U2)
            np.testing.assert_allclose(half, 0.5 * base, rtol=1e-12, atol=1e-12)
        U3 = list(U)
        U3[n] = np.full_like(U[n], 123.0)
        same, _ = oracle_mod.mttkrp(dims, inds, vals, n, U3)
        np.testing.assert_array_equal(same, base)
        perm = np.random.default_rng(n).permutation(vals.shape[0])
        shuf, _ = oracle_mod.mttkrp(dims, inds[:, perm], vals[perm], n, U)
        np.testing.assert_allclose(shuf, base, rtol=1e-12, atol=1e-12)
    # mode permutation: permute tensor modes and the factor list together
    p = [2, 0, 1]
    dims_p = tuple(dims[k] for k in p)
    inds_p = inds[p]
    U_p = [U[k] for k in p]
    for n in range(3):
        a, _ = oracle_mod.mttkrp(dims, inds, vals, p[n], U)
        b, _ = oracle_mod.mttkrp(dims_p, inds_p, vals, n, U_p)
        np.testing.assert_allclose(a, b, rtol=1e-12, atol=1e-12)


def test_sampled_rows_match_full(oracle_mod):
    dims = (64, 50, 40)
    inds, vals = si.powerlaw_coo(dims, 3000, seed=12)
    U = si.factors(dims, 8, seed=1)
    for n in range(3):
        full, fa = oracle_mod.mttkrp(dims, inds, vals, n, U)
        rows = np.array(sorted({0, 1, 5, dims[n] - 1, int(inds[n, 0])}), np.uint32)
        part, pa = oracle_mod.mttkrp_rows(dims, inds, vals, n, U, rows)
        np.testing.assert_array_equal(part, full[rows])
        np.testing.assert_array_equal(pa, fa[rows])


def test_empty_and_degenerate(oracle_mod):
    dims = (5, 6, 7)
    inds = np.zeros((3, 0), np.uint32)
    vals = np.zeros(0, np.float32)
    U = si.factors(dims, 3, seed=0)
    got, ab = oracle_mod.mttkrp(dims, inds, vals, 1, U)
    assert got.shape == (6, 3) and not got.any() and not ab.any()
    # order 1: MTTKRP = the vector itself (empty KRP product)
    inds1 = np.array([[0, 3, 3]], np.uint32)
    vals1 = np.array([1.5, -2.0, 0.25], np.float32)
    got1, _ = oracle_mod.mttkrp((4,), inds1, vals1, 0, [None], R=2)
    np.testing.assert_array_equal(got1[:, 0], [1.5, 0, 0, -1.75])


def test_mode_sort_is_lexicographic_and_stable(oracle_mod):
    dims = (9, 7, 5)
    inds, vals = si.uniform_coo(dims, 200, seed=31)
    # duplicate some coordinates to exercise stability
    inds = np.concatenate([inds, inds[:, :20]], axis=1)
    vals = np.concatenate([vals, -vals[:20]]).astype(np.float32)
    for n in range(3):
        keys = [inds[(n + j) % 3] for j in range(3)]
        order = np.lexsort(keys[::-1])  # numpy lexsort is stable, last key primary
        si_, sv = oracle_mod.mode_sort(inds, vals, n)
        np.testing.assert_array_equal(si_, inds[:, order])
        np.testing.assert_array_equal(sv, vals[order])
