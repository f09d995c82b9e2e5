"""Pins of O-TTM / O-TTV (Eq. 2, Eq. 1) against dense numpy contractions."""
import numpy as np

import synth_inputs as si


def _dense(dims, inds, vals):
    X = np.zeros(dims)
    np.add.at(X, tuple(inds.astype(np.int64)), vals.astype(np.float64))
    return X


def test_ttm_equals_dense_mode_product(oracle_mod):
    dims = (7, 6, 5, 4)
    inds, vals = si.uniform_coo(dims, 300, seed=3)
    X = _dense(dims, inds, vals)
    for n in range(4):
        R = 3
        U = si.factors([dims[n]], R, seed=n)[0]
        fib, Y, Ya = oracle_mod.ttm(dims, inds, vals, n, U)
        # dense n-mode product, R moved to the position of mode n
        Yd = np.moveaxis(np.tensordot(X, U.astype(np.float64), axes=([n], [0])), -1, n)
        others = [k for k in range(4) if k != n]
        # fibers: exactly the distinct coordinate tuples of the other modes, lexicographic
        keys = sorted({tuple(int(inds[k, x]) for k in others) for x in range(vals.shape[0])})
        assert [tuple(int(fib[k, f]) for k in others) for f in range(fib.shape[1])] == keys
        for f, key in enumerate(keys):
            idx = list(key)
            idx.insert(n, slice(None))
            np.testing.assert_allclose(Y[f], Yd[tuple(idx)], rtol=1e-12, atol=1e-12)
        # outside the fibers the dense product is zero (sparse-dense property)
        mask = np.zeros([dims[k] for k in others], bool)
        for key in keys:
            mask[key] = True
        assert np.all(np.moveaxis(Yd, n, -1)[~mask] == 0)
        assert np.all(Ya + 1e-12 >= np.abs(Y))


def test_ttv_is_ttm_with_one_column_and_chains_to_mttkrp(oracle_mod):
    dims = (9, 8, 7)
    inds, vals = si.uniform_coo(dims, 200, seed=5)
    v = si.factors([dims[2]], 1, seed=1)[0][:, 0]
    f1, y1, _ = oracle_mod.ttv(dims, inds, vals, 2, v)
    f2, y2, _ = oracle_mod.ttm(dims, inds, vals, 2, v.reshape(-1, 1))
    np.testing.assert_array_equal(f1, f2)
    np.testing.assert_array_equal(y1, y2[:, 0])
    # (X x_3 c) x_2 b = mode-0 MTTKRP with R = 1 (Eq. 3 with a single column)
    b = si.factors([dims[1]], 1, seed=2)[0][:, 0]
    z = np.zeros(dims[0])
    np.add.at(z, f1[0].astype(np.int64), y1 * b[f1[1]].astype(np.float64))
    U = [None, b.reshape(-1, 1).astype(np.float32), v.reshape(-1, 1).astype(np.float32)]
    m, _ = oracle_mod.mttkrp(dims, inds, vals, 0, U, R=1)
    np.testing.assert_allclose(m[:, 0], z, rtol=1e-12, atol=1e-12)
