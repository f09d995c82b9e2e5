"""Pins of the CP-ALS oracle (oracle/cpals.py), CPU only."""
import itertools

import numpy as np

import synth_inputs as si
from oracle.cpals import cp_als


def _dense_from_cp(lam, U):
    dims = [u.shape[0] for u in U]
    X = np.zeros(dims)
    for r in range(len(lam)):
        t = lam[r]
        for u in U:
            t = np.multiply.outer(t, u[:, r])
        X += t
    return X


def _rank_r_tensor(dims, R, seed):
    rng = np.random.default_rng(seed)
    U = [rng.uniform(0.2, 1.0, size=(d, R)) for d in dims]
    lam = rng.uniform(1.0, 2.0, size=R)
    X = _dense_from_cp(lam, U)
    inds = np.array(list(itertools.product(*[range(d) for d in dims])), dtype=np.uint32).T
    vals = X[tuple(inds)].astype(np.float32)
    return inds, vals


def test_recovers_exact_low_rank_tensor(oracle_mod):
    dims, R = (12, 10, 8), 3
    inds, vals = _rank_r_tensor(dims, R, 1)
    U0 = si.factors(dims, R, seed=3)
    U, lam, fits = cp_als(dims, inds, vals, U0, iters=200, tol=1e-12)
    assert fits[-1] > 0.999, fits[-5:]
    Xhat = _dense_from_cp(lam, [u.astype(np.float64) for u in U])
    X = np.zeros(dims)
    X[tuple(inds)] = vals
    assert np.linalg.norm(X - Xhat) / np.linalg.norm(X) < 2e-3


def _unfold(X, n):
    """Mode-n unfolding, columns with the earliest remaining mode fastest (Kolda-Bader, R#3)."""
    return np.reshape(np.moveaxis(X, n, 0), (X.shape[n], -1), order="F")


def _krp(mats):
    """Khatri-Rao product (Eq. 4): column r = kron(mats[0][:, r], mats[1][:, r], ...)."""
    out = mats[0]
    for m in mats[1:]:
        out = np.einsum("ir,jr->ijr", out, m).reshape(-1, out.shape[1])
    return out


def test_each_update_is_the_dense_least_squares_solution(oracle_mod):
    """Every ALS update U_n = argmin ||X_(n) - U_n KRP^T||_F (Kolda-Bader), solved here by
    np.linalg.lstsq on the dense unfolding and the explicit Khatri-Rao product -- a formulation
    that shares neither the MTTKRP nor the normal equations with the oracle."""
    dims, R = (15, 12, 9, 7), 4
    inds, vals = si.uniform_coo(dims, 600, seed=2)
    X = np.zeros(dims)
    X[tuple(inds)] = vals
    rec = []
    U0 = si.factors(dims, R, seed=4)
    cp_als(dims, inds, vals, U0, iters=2, record=rec)
    # replay: the factors the oracle held before each update (fp32 storage, as the oracle)
    cur = [u.astype(np.float32) for u in U0]
    for n, M, V, Un in rec:
        others = [cur[k].astype(np.float64) for k in reversed(range(len(dims))) if k != n]
        K = _krp(others)  # rows ordered with the earliest remaining mode fastest
        ls = np.linalg.lstsq(K, _unfold(X, n).T, rcond=None)[0].T
        assert np.allclose(Un, ls, rtol=1e-7, atol=1e-9 * np.abs(ls).max()), n
        lam = np.sqrt(np.sum(Un * Un, axis=0))
        lam[lam == 0] = 1.0
        cur[n] = (Un / lam).astype(np.float32)


def test_fit_formula_matches_dense_reconstruction(oracle_mod):
    dims, R = (9, 8, 7), 3
    inds, vals = si.uniform_coo(dims, 200, seed=5)
    X = np.zeros(dims)
    X[tuple(inds)] = vals
    for iters in (1, 2, 5):
        U, lam, fits = cp_als(dims, inds, vals, si.factors(dims, R, seed=6), iters=iters)
        Xhat = _dense_from_cp(lam, [u.astype(np.float64) for u in U])
        brute = 1.0 - np.linalg.norm(X - Xhat) / np.linalg.norm(X)
        assert abs(brute - fits[-1]) < 1e-6


def test_fit_is_monotone(oracle_mod):
    dims, R = (30, 25, 20), 5
    inds, vals = si.powerlaw_coo(dims, 3000, seed=7)
    _, _, fits = cp_als(dims, inds, vals, si.factors(dims, R, seed=8), iters=15)
    assert all(b >= a - 1e-6 for a, b in zip(fits, fits[1:])), fits
