"""Pins of the oracle's TEW / TS (single precision).

* TS and same-pattern TEW against numpy float32 arithmetic (an independent IEEE fp32
  implementation), bit for bit, for every operator, including signed zeros, infinities and
  subnormals;
* closed forms: x - x = 0, x * 1 = x, x + 0 = x, x / x = 1 (x finite, nonzero), 2x exact;
* different patterns (R#31): against a pure-Python dictionary merge on small tensors, the
  output pattern sizes against numpy set operations (|X u Y| for add/sub, |X n Y| for
  mul/div), and a repeated coordinate inside one input is rejected.
"""
import numpy as np
import pytest

import synth_inputs as si

OPS = {"add": np.add, "sub": np.subtract, "mul": np.multiply, "div": np.divide}


def _bits(a):
    return np.asarray(a, np.float32).view(np.uint32)


def _special_values(n, seed):
    rng = np.random.default_rng(seed)
    v = rng.uniform(-1, 1, n).astype(np.float32)
    v[:8] = np.array([0.0, -0.0, np.inf, -np.inf, 1e-40, -1e-40, 3.4e38, 1.0], np.float32)
    return v


@pytest.mark.parametrize("op", list(OPS))
def test_ts_matches_numpy_float32(oracle_mod, op):
    v = _special_values(5000, 1)
    for s in (np.float32(0.75), np.float32(-3.0e-39), np.float32(1e30)):
        got = oracle_mod.ts(v, op, s)
        with np.errstate(all="ignore"):
            ref = OPS[op](v, s).astype(np.float32)
        nan = np.isnan(ref)
        assert np.array_equal(np.isnan(got), nan)
        np.testing.assert_array_equal(_bits(got)[~nan], _bits(ref)[~nan])


@pytest.mark.parametrize("op", list(OPS))
def test_tew_same_matches_numpy_float32(oracle_mod, op):
    a = _special_values(5000, 2)
    b = _special_values(5000, 3)[::-1].copy()
    got = oracle_mod.tew_same(a, b, op)
    with np.errstate(all="ignore"):
        ref = OPS[op](a, b).astype(np.float32)
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(got), nan)
    np.testing.assert_array_equal(_bits(got)[~nan], _bits(ref)[~nan])


def test_closed_forms(oracle_mod):
    x = np.random.default_rng(4).uniform(-1, 1, 10000).astype(np.float32)
    x[x == 0] = 0.5
    assert np.all(oracle_mod.tew_same(x, x, "sub") == 0)
    np.testing.assert_array_equal(_bits(oracle_mod.ts(x, "mul", 1.0)), _bits(x))
    np.testing.assert_array_equal(_bits(oracle_mod.ts(x, "add", 0.0)), _bits(x))
    assert np.all(oracle_mod.tew_same(x, x, "div") == 1)
    np.testing.assert_array_equal(oracle_mod.tew_same(x, x, "add"), x * np.float32(2))


def _dict_merge(ix, vx, iy, vy, op):
    X = {tuple(int(c) for c in ix[:, i]): vx[i] for i in range(ix.shape[1])}
    Y = {tuple(int(c) for c in iy[:, i]): vy[i] for i in range(iy.shape[1])}
    keys = sorted(set(X) | set(Y)) if op in ("add", "sub") else sorted(set(X) & set(Y))
    out = []
    for k in keys:
        if k in X and k in Y:
            z = OPS[op](np.float32(X[k]), np.float32(Y[k]))
        elif k in X:
            z = np.float32(X[k])
        else:
            z = np.float32(0) - np.float32(Y[k]) if op == "sub" else np.float32(Y[k])
        out.append((k, np.float32(z)))
    return out


@pytest.mark.parametrize("op", list(OPS))
def test_merge_matches_dict_reference(oracle_mod, op):
    dims = (30, 20, 10)
    ix, vx = si.uniform_coo(dims, 800, seed=5)
    iy, vy = si.uniform_coo(dims, 600, seed=6)
    vy[vy == 0] = 0.25
    zi, zv = oracle_mod.tew_merge(ix, vx, iy, vy, op)
    ref = _dict_merge(ix, vx, iy, vy, op)
    assert zi.shape[1] == len(ref)
    for j, (k, z) in enumerate(ref):
        assert tuple(int(c) for c in zi[:, j]) == k
        assert _bits(zv[j]) == _bits(z)
    sx = {tuple(c) for c in ix.T.tolist()}
    sy = {tuple(c) for c in iy.T.tolist()}
    assert zi.shape[1] == (len(sx | sy) if op in ("add", "sub") else len(sx & sy))


def test_merge_edge_cases(oracle_mod):
    dims = (5, 5)
    ix = np.array([[0, 1], [2, 3]], np.uint32)
    vx = np.array([1.0, 2.0], np.float32)
    e = np.zeros((2, 0), np.uint32)
    zi, zv = oracle_mod.tew_merge(ix, vx, e, np.zeros(0, np.float32), "sub")
    np.testing.assert_array_equal(zi, ix)
    zi, zv = oracle_mod.tew_merge(e, np.zeros(0, np.float32), ix, vx, "sub")
    np.testing.assert_array_equal(zv, -vx)
    zi, zv = oracle_mod.tew_merge(ix, vx, e, np.zeros(0, np.float32), "mul")
    assert zi.shape[1] == 0
    dup = np.array([[0, 0], [2, 2]], np.uint32)
    with pytest.raises(ValueError):
        oracle_mod.tew_merge(dup, vx, ix, vx, "add")
