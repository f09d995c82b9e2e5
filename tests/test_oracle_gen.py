"""Pins of the oracle's Stochastic-Kronecker generator (R#19-R#23).

The paper prints no initiator and no generated tensor, so the pins are
statistical closed forms plus structural guarantees:
  * product-form initiator (q per mode per level) => popcount(i_k) ~ Binomial(L, 1-q);
  * a general 2^N initiator => each level's bit tuple follows the table;
  * q = 0.5 => uniform over the valid box (stripping keeps uniformity);
  * exact M, distinct coordinates, in-range, lexicographic order, determinism,
    first-draw semantics (a smaller M is a subset with the same values).
"""
import numpy as np
import pytest
from scipy import stats


def _popcount(a):
    a = a.astype(np.uint64)
    c = np.zeros_like(a)
    for b in range(32):
        c += (a >> np.uint64(b)) & np.uint64(1)
    return c.astype(np.int64)


def test_structure_and_determinism(oracle_mod):
    dims = (12092, 9184, 28818)
    inds, vals = oracle_mod.gen_powerlaw(dims, 30000, seed=1002)
    assert inds.shape == (3, 30000) and vals.shape == (30000,)
    for k in range(3):
        assert inds[k].max() < dims[k]
    keys = [tuple(inds[:, x]) for x in range(inds.shape[1])]
    assert len(set(keys)) == len(keys)
    assert keys == sorted(keys)
    assert vals.min() >= -1.0 and vals.max() < 1.0
    inds2, vals2 = oracle_mod.gen_powerlaw(dims, 30000, seed=1002)
    np.testing.assert_array_equal(inds, inds2)
    np.testing.assert_array_equal(vals.view(np.uint32), vals2.view(np.uint32))
    inds3, _ = oracle_mod.gen_powerlaw(dims, 30000, seed=1003)
    assert not np.array_equal(inds, inds3)


def test_first_draw_semantics(oracle_mod):
    dims = (64, 64, 64)  # small box => many repeated draws
    big_i, big_v = oracle_mod.gen_powerlaw(dims, 5000, seed=7)
    small_i, small_v = oracle_mod.gen_powerlaw(dims, 1000, seed=7)
    big = {tuple(big_i[:, x]): big_v[x] for x in range(big_i.shape[1])}
    for x in range(small_i.shape[1]):
        key = tuple(small_i[:, x])
        assert key in big and big[key] == small_v[x]


def test_popcount_is_binomial(oracle_mod):
    L = 12
    dims = (1 << L,) * 3
    q = 0.75
    inds, _ = oracle_mod.gen_powerlaw(dims, 20000, seed=5, q=q)
    p = stats.binom.pmf(np.arange(L + 1), L, 1 - q)
    for k in range(3):
        obs = np.bincount(_popcount(inds[k]), minlength=L + 1)
        exp = p * inds.shape[1]
        keep = exp >= 5
        o = np.append(obs[keep], obs[~keep].sum())
        e = np.append(exp[keep], exp[~keep].sum())
        chi2 = ((o - e) ** 2 / e).sum()
        assert stats.chi2.sf(chi2, len(o) - 1) > 1e-4, (k, obs, exp)
    # modes are independent under a product-form initiator
    tab = np.zeros((2, 2))
    np.add.at(tab, (inds[0] & 1, inds[1] & 1), 1)
    assert stats.chi2_contingency(tab)[1] > 1e-4


def test_general_initiator_level_distribution(oracle_mod):
    T = np.array([0.57, 0.19, 0.19, 0.05])  # Graph500 2x2 initiator (P:372 lineage)
    L = 16
    inds, _ = oracle_mod.gen_powerlaw((1 << L, 1 << L), 5000, seed=3, initiator=T)
    for lvl in (0, 7, 15):
        cell = ((inds[0] >> lvl) & 1) + 2 * ((inds[1] >> lvl) & 1)
        obs = np.bincount(cell, minlength=4)
        chi2 = ((obs - T * obs.sum()) ** 2 / (T * obs.sum())).sum()
        assert stats.chi2.sf(chi2, 3) > 1e-4, (lvl, obs)


def test_half_is_uniform_with_stripping(oracle_mod):
    dims = (100, 100, 100)  # not powers of two: draws outside are stripped
    inds, _ = oracle_mod.gen_powerlaw(dims, 10000, seed=1001, q=0.5)
    for k in range(3):
        obs = np.bincount(inds[k] // 10, minlength=10)
        assert stats.chisquare(obs).pvalue > 1e-4


def test_degenerate_initiators(oracle_mod):
    T = np.zeros(8)
    T[7] = 1.0  # all mass on the all-ones cell => the single coordinate (2^L_k - 1)_k
    inds, _ = oracle_mod.gen_powerlaw((8, 16, 4), 1, seed=1, initiator=T)
    assert list(inds[:, 0]) == [7, 15, 3]
    with pytest.raises(ValueError):
        oracle_mod.gen_powerlaw((8, 16, 4), 2, seed=1, initiator=T)
    with pytest.raises(ValueError):  # more nonzeros than cells
        oracle_mod.gen_powerlaw((2, 2), 5, seed=1)
    inds0, vals0 = oracle_mod.gen_powerlaw((5, 5), 0, seed=1)
    assert inds0.shape == (2, 0) and vals0.shape == (0,)
    # the full box: every cell exactly once
    inds4, _ = oracle_mod.gen_powerlaw((3, 5), 15, seed=2)
    assert sorted(map(tuple, inds4.T)) == [(i, j) for i in range(3) for j in range(5)]


def test_label_permutation_is_a_bijection_per_mode(oracle_mod):
    """R#22 (permute = 1): pi_k is a bijection of [0, I_k) for powers of two, their
    neighbours and odd sizes; different modes / seeds give different permutations."""
    for dim in (1, 2, 3, 7, 64, 127, 128, 129, 1000, 4097):
        img = [oracle_mod.relabel_index(v, dim, 11, 2) for v in range(dim)]
        assert sorted(img) == list(range(dim)), dim
    a = [oracle_mod.relabel_index(v, 1000, 11, 0) for v in range(1000)]
    b = [oracle_mod.relabel_index(v, 1000, 11, 1) for v in range(1000)]
    c = [oracle_mod.relabel_index(v, 1000, 12, 0) for v in range(1000)]
    assert a != b and a != c and a != list(range(1000))


def test_permuted_generator_keeps_the_row_count_multiset(oracle_mod):
    """Relabelling moves rows but keeps every row's nonzeros: the sorted row counts of every
    mode, the multiset of values and uniqueness are those of the unpermuted tensor, and the
    permuted tensor is lexicographically sorted."""
    dims, M, seed = (300, 200, 500), 20_000, 9
    i0, v0 = oracle_mod.gen_powerlaw(dims, M, seed)
    i1, v1 = oracle_mod.gen_powerlaw(dims, M, seed, permute=True)
    for k, d in enumerate(dims):
        assert np.array_equal(np.sort(np.bincount(i0[k], minlength=d)), np.sort(np.bincount(i1[k], minlength=d)))
        # pi_k applied to the unpermuted coordinates gives exactly the permuted ones
        mapped = np.array([oracle_mod.relabel_index(v, d, seed, k) for v in range(d)], np.uint32)[i0[k]]
        assert np.array_equal(np.sort(mapped), np.sort(i1[k]))
    assert np.array_equal(np.sort(v0.view(np.uint32)), np.sort(v1.view(np.uint32)))
    key = (i1[0].astype(np.int64) * dims[1] + i1[1]) * dims[2] + i1[2]
    assert np.all(np.diff(key) > 0)
