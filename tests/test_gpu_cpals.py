"""CP-ALS on the GPU against the fp64 CP-ALS oracle (oracle/cpals.py) from
the same initial factors, plus its building blocks against numpy."""
import itertools

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


def test_building_blocks(env):
    pasta, oracle, torch = env
    rng = np.random.default_rng(0)
    for R in (1, 5, 16, 32, 64):
        U = rng.uniform(-1, 1, size=(5000, R)).astype(np.float32)
        Ut = torch.from_numpy(U).cuda()
        G = pasta.pasta_gram(Ut).cpu().numpy()
        ref = U.astype(np.float64).T @ U.astype(np.float64)
        # per 64-row tile in fp32, tiles combined in fp64
        assert np.allclose(G, ref, rtol=1e-5, atol=1e-5 * np.abs(ref).max())
        grams = [pasta.pasta_gram(torch.from_numpy(rng.uniform(0, 1, (300, R)).astype(np.float32)).cuda())
                 for _ in range(2)]
        M = rng.uniform(-1, 1, size=(700, R)).astype(np.float32)
        Uo, colsq = pasta.pasta_cpals_solve(torch.from_numpy(M).cuda(), grams)
        V = grams[0].cpu().numpy() * grams[1].cpu().numpy()
        Uref = np.linalg.solve(V.T, M.astype(np.float64).T).T
        got = Uo.cpu().numpy().astype(np.float64)
        assert np.allclose(got, Uref, rtol=1e-4, atol=1e-5 * np.abs(Uref).max()), R
        assert np.allclose(colsq.cpu().numpy(), np.sum(got ** 2, axis=0), rtol=1e-5)
        lam = pasta.pasta_normalize_columns(Uo, colsq).cpu().numpy()
        assert np.allclose(lam, np.sqrt(np.sum(got ** 2, axis=0)), rtol=1e-6)
        assert np.allclose(np.linalg.norm(Uo.cpu().numpy().astype(np.float64), axis=0), 1.0, atol=1e-5)


def test_gram_many_tiles_per_cta(env):
    """The gram and factor-update kernels' persistent CTAs walk several double-buffered
    (cp.async) row tiles each (rows well above 148 x 8 tiles) and a ragged last tile, for every
    tiled rank."""
    pasta, oracle, torch = env
    rng = np.random.default_rng(3)
    for R, rows in ((4, 5_000_011), (8, 2_500_007), (16, 700_001), (32, 400_003), (64, 200_009)):
        U = rng.uniform(-1, 1, size=(rows, R)).astype(np.float32)
        G = pasta.pasta_gram(torch.from_numpy(U).cuda()).cpu().numpy()
        U64 = U.astype(np.float64)
        ref = U64.T @ U64
        assert np.allclose(G, ref, rtol=1e-5, atol=1e-6 * np.abs(ref).max()), R
        # the factor update U = M Wn walks the same double-buffered tiles
        W = rng.uniform(-1, 1, size=(R, R)).astype(np.float32)
        got = pasta.pasta_rows_times(torch.from_numpy(U).cuda(), torch.from_numpy(W).cuda()).cpu().numpy()
        want = U64 @ W.astype(np.float64)
        assert np.allclose(got, want, rtol=1e-5, atol=1e-5 * R), R


def test_fused_update_blocks(env):
    """pasta_cpals_prepare + pasta_rows_times == solve -> normalise -> gram (numpy fp64)."""
    pasta, oracle, torch = env
    rng = np.random.default_rng(1)
    for R in (1, 7, 16, 32, 64):
        grams = [pasta.pasta_gram(torch.from_numpy(rng.uniform(0, 1, (400, R)).astype(np.float32)).cuda())
                 for _ in range(2)]
        M = rng.uniform(-1, 1, size=(3000, R)).astype(np.float32)
        Md = torch.from_numpy(M).cuda()
        GM = pasta.pasta_gram(Md)
        Wn, Gn, lam = pasta.pasta_cpals_prepare(GM, grams)
        U = pasta.pasta_rows_times(Md, Wn).cpu().numpy().astype(np.float64)
        V = grams[0].cpu().numpy() * grams[1].cpu().numpy()
        Uref = np.linalg.solve(V.T, M.astype(np.float64).T).T
        lref = np.linalg.norm(Uref, axis=0)
        assert np.allclose(lam.cpu().numpy(), lref, rtol=1e-4), R
        Un = Uref / lref
        assert np.allclose(U, Un, rtol=1e-3, atol=1e-4 * np.abs(Un).max()), R
        assert np.allclose(Gn.cpu().numpy(), Un.T @ Un, atol=1e-4), R


@pytest.mark.parametrize("fused", ["1", "0"])
@pytest.mark.parametrize("dims,nnz,R,iters", [((60, 50, 40), 8000, 8, 1), ((60, 50, 40), 8000, 8, 3),
                                               ((40, 30, 20, 10), 6000, 16, 2)])
def test_cpals_matches_oracle(env, dims, nnz, R, iters, fused, monkeypatch):
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_CPALS_FUSED", fused)
    from oracle.cpals import cp_als
    inds, vals = si.powerlaw_coo(dims, nnz, seed=nnz + R)
    U0 = si.factors(dims, R, seed=R)
    Uo, lam_o, fits_o = cp_als(dims, inds, vals, U0, iters=iters)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    Ud = [torch.from_numpy(u.copy()).cuda() for u in U0]
    lam, fits, it = pasta.pasta_cpals_coo(x, Ud, max_iters=iters, tol=0.0)
    assert it == iters
    assert np.allclose(fits, fits_o, atol=2e-4), (fits, fits_o)
    assert np.allclose(lam, lam_o, rtol=2e-3)
    for k in range(len(dims)):
        g, o = Ud[k].cpu().numpy(), Uo[k]
        assert np.abs(g - o).max() < 2e-3 * np.abs(o).max() + 1e-5, k


def test_cpals_recovers_low_rank(env):
    pasta, oracle, torch = env
    rng = np.random.default_rng(3)
    dims, R = (30, 25, 20), 4
    A = [rng.uniform(0.2, 1.0, size=(d, R)) for d in dims]
    X = np.einsum("ir,jr,kr->ijk", *A)
    inds = np.array(list(itertools.product(*[range(d) for d in dims])), dtype=np.uint32).T
    vals = X[tuple(inds)].astype(np.float32)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    Ud = [torch.from_numpy(u).cuda() for u in si.factors(dims, R, seed=9)]
    lam, fits, it = pasta.pasta_cpals_coo(x, Ud, max_iters=300, tol=1e-9)
    assert fits[-1] > 0.995, fits[-3:]
    # ALS is monotone; near fit = 1 the fit formula cancels (||X||^2 + ||Xhat||^2 - 2<X,Xhat>),
    # so only the first sweeps are compared, with a tolerance for fp32 factor storage
    head = fits[:10]
    assert all(b >= a - 1e-3 for a, b in zip(head, head[1:])), head


def test_row_partitioned_cpals_single_process_matches(env):
    """RowPartitionedCPALS with world = 1 (no process group) equals pasta_cpals_coo."""
    pasta, oracle, torch = env
    from paper_conf_iiswc_lilwlob20_b200.parallel import RowPartitionedCPALS
    dims, R = (200, 150, 100), 8
    inds, vals = si.powerlaw_coo(dims, 20000, seed=4)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    U0 = si.factors(dims, R, seed=2)
    Ua = [torch.from_numpy(u.copy()).cuda() for u in U0]
    Ub = [torch.from_numpy(u.copy()).cuda() for u in U0]
    lam_a, fits_a, _ = pasta.pasta_cpals_coo(x, Ua, max_iters=4, tol=0.0)
    runner = RowPartitionedCPALS(x, 0, 1, R, torch.device("cuda"))
    lam_b, fits_b = runner.run(Ub, max_iters=4, tol=0.0)
    assert np.allclose(fits_a, fits_b, atol=1e-6)
    assert np.allclose(lam_a, lam_b, rtol=1e-5)
