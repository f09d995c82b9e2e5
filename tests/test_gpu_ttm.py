"""TTV / TTM on the GPU against the oracle (Eq. 1, Eq. 2):
fibers bit-exact, values within 1e-4 * sum|terms| + 1e-6."""
import numpy as np
import pytest

import synth_inputs as si

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env(oracle_mod):
    import torch

    import paper_conf_iiswc_lilwlob20_b200 as pasta
    assert torch.cuda.is_available()
    torch.cuda.set_device(0)
    return pasta, oracle_mod, torch


@pytest.mark.parametrize("dims,nnz,R", [((300, 200, 500), 50_013, 16), ((60, 70, 80, 90), 40_007, 8),
                                        ((1000, 900), 30_001, 3), ((4096, 4096, 4096), 200_000, 32)])
def test_ttm_and_ttv_match_oracle(env, dims, nnz, R):
    pasta, oracle, torch = env
    inds, vals = si.powerlaw_coo(dims, nnz, seed=nnz)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    for n in range(len(dims)):
        U = si.factors([dims[n]], R, seed=n + R)[0]
        fib, Y, Ya = oracle.ttm(dims, inds, vals, n, U)
        assert pasta.pasta_coo_fibers(x, n) == fib.shape[1]
        gf = pasta.pasta_coo_fiber_export(x, n)
        for k in range(len(dims)):
            if k != n:
                np.testing.assert_array_equal(gf[k], fib[k])
        got = pasta.pasta_ttm_coo(x, n, torch.from_numpy(U).cuda()).cpu().numpy().astype(np.float64)
        assert np.all(np.abs(got - Y) <= 1e-4 * Ya + 1e-6), (dims, n)
        v = U[:, 0].copy()
        fv, yv, yva = oracle.ttv(dims, inds, vals, n, v)
        gv = pasta.pasta_ttv_coo(x, n, torch.from_numpy(v).cuda()).cpu().numpy().astype(np.float64)
        assert np.all(np.abs(gv - yv) <= 1e-4 * yva + 1e-6)


def test_ttm_hot_fiber_and_empty(env):
    pasta, oracle, torch = env
    dims = (50, 4000, 30)
    # one mode-1 fiber holds 3000 nonzeros (all of (i0=7, i2=3) with distinct i1)
    i1 = np.random.default_rng(0).choice(4000, 3000, replace=False).astype(np.uint32)
    hot = np.stack([np.full(3000, 7, np.uint32), i1, np.full(3000, 3, np.uint32)])
    rest, _ = si.uniform_coo(dims, 5000, seed=2)
    keep = ~((rest[0] == 7) & (rest[2] == 3))
    inds = np.ascontiguousarray(np.concatenate([hot, rest[:, keep]], axis=1))
    vals = np.random.default_rng(1).uniform(-1, 1, inds.shape[1]).astype(np.float32)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    U = si.factors([dims[1]], 16, seed=3)[0]
    fib, Y, Ya = oracle.ttm(dims, inds, vals, 1, U)
    got = pasta.pasta_ttm_coo(x, 1, torch.from_numpy(U).cuda()).cpu().numpy().astype(np.float64)
    assert np.all(np.abs(got - Y) <= 1e-4 * Ya + 1e-6)
    # TTV's warp-segmented sum: the 3000-entry fiber spans many 128-entry tiles
    v = U[:, 0].copy()
    fv, yv, yva = oracle.ttv(dims, inds, vals, 1, v)
    gv = pasta.pasta_ttv_coo(x, 1, torch.from_numpy(v).cuda()).cpu().numpy().astype(np.float64)
    assert np.all(np.abs(gv - yv) <= 1e-4 * yva + 1e-6)
    e = pasta.pasta_coo_from_arrays(dims, np.zeros((3, 0), np.uint32), np.zeros(0, np.float32))
    assert pasta.pasta_coo_fibers(e, 0) == 0


@pytest.mark.parametrize("M,maxlen,seed", [(1, 1, 0), (127, 3, 1), (129, 200, 2), (100_003, 9, 3),
                                           (300_001, 700, 4), (65_536, 1, 5)])
def test_ttv_segmented_sum_run_lengths(env, M, maxlen, seed):
    """Order-2 tensors whose mode-0 fibers (rows of X^T) have lengths 1..maxlen: fibers start
    and end at every position relative to lanes and 128-entry tiles."""
    pasta, oracle, torch = env
    rng = np.random.default_rng(seed)
    lens = []
    tot = 0
    while tot < M:
        l = int(min(rng.integers(1, maxlen + 1), M - tot))
        lens.append(l)
        tot += l
    nf = len(lens)
    J = max(maxlen, 1) + 5
    i1 = np.repeat(np.arange(nf, dtype=np.uint32), lens)
    i0 = np.concatenate([rng.choice(J, l, replace=False) for l in lens]).astype(np.uint32)
    inds = np.ascontiguousarray(np.stack([i0, i1]))
    vals = rng.uniform(-1, 1, M).astype(np.float32)
    dims = (J, nf)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    v = rng.uniform(0, 1, J).astype(np.float32)
    fv, yv, yva = oracle.ttv(dims, inds, vals, 0, v)
    gv = pasta.pasta_ttv_coo(x, 0, torch.from_numpy(v).cuda()).cpu().numpy().astype(np.float64)
    assert gv.shape == yv.shape
    assert np.all(np.abs(gv - yv) <= 1e-4 * yva + 1e-6)
