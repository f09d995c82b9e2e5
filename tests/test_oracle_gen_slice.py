"""Pins of the oracle's FireHose-style slice power-law generator (P:225,
P:229; reading R#30: every mode index independently from P(i) ~ (i+1)^-alpha).

The paper prints neither the generator's parameters nor its output, so the pins are the
closed-form marginal (chi-square against the normalised (i+1)^-alpha law, computed here
with numpy, on boxes where repeated coordinates are negligible), its special cases
(alpha = 0 is uniform; the head ratio P(0)/P(1) = 2^alpha), independence of the modes, and
the structural guarantees shared with the Kronecker generator (exact M, distinct,
in-range, lexicographic, deterministic, first-draw semantics).
"""
import numpy as np
import pytest
from scipy import stats


def _chi2_p(obs, p):
    exp = p * obs.sum()
    keep = exp >= 5
    o = np.append(obs[keep], obs[~keep].sum())
    e = np.append(exp[keep], exp[~keep].sum())
    if e[-1] == 0:
        o, e = o[:-1], e[:-1]
    return stats.chisquare(o, e).pvalue


@pytest.mark.parametrize("alpha", [0.0, 0.5, 0.7, 1.0])
def test_marginal_is_power_law(oracle_mod, alpha):
    # four modes, three huge: repeated coordinates (which the generator drops) are < 1e-3 of
    # the draws for alpha <= 1, below the chi-square resolution
    dims = (60, 1 << 20, 1 << 20, 1 << 20)
    inds, _ = oracle_mod.gen_slice_powerlaw(dims, 40000, seed=3, alpha=alpha)
    i = np.arange(dims[0], dtype=np.float64)
    p = (i + 1.0) ** (-alpha)
    p /= p.sum()
    obs = np.bincount(inds[0], minlength=dims[0])
    assert _chi2_p(obs, p) > 1e-3
    # a large mode: compare the first 64 bins + the tail mass
    big = np.arange(dims[1], dtype=np.float64)
    pb = (big + 1.0) ** (-alpha)
    pb /= pb.sum()
    ob = np.bincount(inds[1], minlength=dims[1]).astype(np.float64)
    obs2 = np.append(ob[:64], ob[64:].sum())
    p2 = np.append(pb[:64], pb[64:].sum())
    assert _chi2_p(obs2, p2) > 1e-3


def test_alpha_zero_is_uniform_and_modes_independent(oracle_mod):
    dims = (16, 16, 1 << 16)
    inds, _ = oracle_mod.gen_slice_powerlaw(dims, 20000, seed=9, alpha=0.0)
    table = np.zeros((16, 16))
    np.add.at(table, (inds[0], inds[1]), 1)
    assert stats.chisquare(table.ravel()).pvalue > 1e-3  # uniform joint of modes 0, 1
    inds, _ = oracle_mod.gen_slice_powerlaw(dims, 20000, seed=9, alpha=1.0)
    table = np.zeros((16, 16))
    np.add.at(table, (inds[0], inds[1]), 1)
    assert stats.chi2_contingency(table).pvalue > 1e-3  # independence


def test_head_ratio(oracle_mod):
    alpha = 1.0  # P(0) / P(1) = 2^alpha; < 0.5 % of the draws repeat in this box
    inds, _ = oracle_mod.gen_slice_powerlaw((8, 1 << 20, 1 << 20, 1 << 20), 60000, seed=5, alpha=alpha)
    c = np.bincount(inds[0], minlength=8)
    ratio = c[0] / c[1]
    assert abs(ratio - 2 ** alpha) < 0.1


def test_structure_determinism_first_draw(oracle_mod):
    dims = (32768, 32768, 76)  # irrS-shaped (Table II s4)
    inds, vals = oracle_mod.gen_slice_powerlaw(dims, 20000, seed=4)
    assert inds.shape == (3, 20000)
    keys = [tuple(inds[:, x]) for x in range(inds.shape[1])]
    assert len(set(keys)) == len(keys) and keys == sorted(keys)
    for k in range(3):
        assert inds[k].max() < dims[k]
    assert set(np.unique(inds[2])) == set(range(76))  # the small mode is completely dense
    i2, v2 = oracle_mod.gen_slice_powerlaw(dims, 20000, seed=4)
    np.testing.assert_array_equal(inds, i2)
    np.testing.assert_array_equal(vals.view(np.uint32), v2.view(np.uint32))
    small_i, small_v = oracle_mod.gen_slice_powerlaw(dims, 3000, seed=4)
    big = {tuple(inds[:, x]): vals[x] for x in range(inds.shape[1])}
    for x in range(small_i.shape[1]):
        assert big[tuple(small_i[:, x])] == small_v[x]
    # saturated small box: every cell, exactly once
    full, _ = oracle_mod.gen_slice_powerlaw((4, 5, 3), 60, seed=1, alpha=1.0)
    assert full.shape[1] == 60 and len({tuple(full[:, x]) for x in range(60)}) == 60


def test_invalid(oracle_mod):
    with pytest.raises(ValueError):
        oracle_mod.gen_slice_powerlaw((4, 4), 17, seed=1)
    with pytest.raises(ValueError):
        oracle_mod.gen_slice_powerlaw((4, 4), 3, seed=1, alpha=-1.0)
