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


U32 = 2.0 ** -24  # fp32 unit roundoff


def gamma(k):
    """gamma_k = k u / (1 - k u): bound on the relative error of k fp32 roundings (Higham)."""
    return k * U32 / (1.0 - k * U32)


def assert_gram_within_bound(G, U, what=""):
    """pasta_gram accumulates <= 64 rows per fp32 partial (FMA: one rounding per row) and
    combines partials in fp64, so |G - U^T U| <= gamma_64 (|U|^T |U|) elementwise (DESIGN.md
    R#33); the fp64 combination adds < 1e-12 relative."""
    U64 = np.asarray(U, np.float64)
    ref = U64.T @ U64
    bound = gamma(64) * (np.abs(U64).T @ np.abs(U64)) * (1 + 1e-12) + 1e-300
    err = np.abs(np.asarray(G, np.float64) - ref)
    assert np.all(err <= bound), f"{what}: gram error {np.max(err / bound):.3f} x the bound"


U64E = 2.0 ** -53  # fp64 unit roundoff


def inverse_error(V):
    """Normwise bound on the error of the library's R x R inverse (fp64 Gauss-Jordan with
    partial pivoting plus a ridge of 1e-14 tr(V) / R, cpals.cu hadamard_inverse):
    ||dW||_2 <= (4 R u64 kappa_2(V) + rho ||W||_2) ||W||_2  (first order; R#33)."""
    R = V.shape[0]
    W = np.linalg.inv(V)
    nw = np.linalg.norm(W, 2)
    rho = 1e-14 * max(np.trace(V), 1.0) / R
    return (4 * R * U64E * np.linalg.cond(V) + rho * nw) * nw, W


def test_building_blocks(env):
    """Each stage against the exact fp64 function of its own (GPU) inputs, within the stage's
    rounding bound (R#33): gram gamma_64; solve = fp64 inverse (inverse_error) + fp32 output
    rounding; colsq / lambda / normalisation in fp64 of the fp32 factor."""
    pasta, oracle, torch = env
    rng = np.random.default_rng(0)
    for R in (1, 5, 16, 32, 64):
        U = rng.uniform(-1, 1, size=(5000, R)).astype(np.float32)
        Ut = torch.from_numpy(U).cuda()
        assert_gram_within_bound(pasta.pasta_gram(Ut).cpu().numpy(), U, f"R={R}")
        grams = [pasta.pasta_gram(torch.from_numpy(rng.uniform(0, 1, (300, R)).astype(np.float32)).cuda())
                 for _ in range(2)]
        M = rng.uniform(-1, 1, size=(700, R)).astype(np.float32)
        Uo, colsq = pasta.pasta_cpals_solve(torch.from_numpy(M).cuda(), grams)
        V = grams[0].cpu().numpy() * grams[1].cpu().numpy()
        dW, W = inverse_error(V)
        M64 = M.astype(np.float64)
        Uref = M64 @ W
        got = Uo.cpu().numpy().astype(np.float64)
        # W rounded to fp32 (one rounding), then R fp32 FMAs per element
        tol = gamma(R + 1) * (np.abs(M64) @ np.abs(W)) + 2 * np.linalg.norm(M64, axis=1, keepdims=True) * dW
        assert np.all(np.abs(got - Uref) <= tol + 1e-300), (R, np.max(np.abs(got - Uref) / tol))
        # colsq: fp32 FMA sums of x^2 per thread (at most `rows` terms), fp64 across threads
        rows = M.shape[0]
        ref_cs = np.sum(got ** 2, axis=0)
        assert np.all(np.abs(colsq.cpu().numpy() - ref_cs) <= gamma(rows + 1) * ref_cs), R
        lam = pasta.pasta_normalize_columns(Uo, colsq).cpu().numpy()
        assert np.allclose(lam, np.sqrt(colsq.cpu().numpy()), rtol=4 * U64E, atol=0)
        # normalised fp32 columns: colsq's bound halves under the sqrt, plus one rounding each
        assert np.allclose(np.linalg.norm(Uo.cpu().numpy().astype(np.float64), axis=0), 1.0,
                           atol=gamma(rows + 1) / 2 + 4 * U32)


def test_gram_many_tiles_per_cta(env):
    """The gram and factor-update kernels' persistent CTAs walk several double-buffered
    (cp.async) row tiles each (rows well above 148 x 8 tiles) and a ragged last tile, for every
    tiled rank."""
    pasta, oracle, torch = env
    rng = np.random.default_rng(3)
    for R, rows in ((4, 5_000_011), (8, 2_500_007), (16, 700_001), (32, 400_003), (64, 200_009)):
        U = rng.uniform(-1, 1, size=(rows, R)).astype(np.float32)
        assert_gram_within_bound(pasta.pasta_gram(torch.from_numpy(U).cuda()).cpu().numpy(), U, f"R={R}")
        U64 = U.astype(np.float64)
        # the factor update U = M Wn walks the same double-buffered tiles
        W = rng.uniform(-1, 1, size=(R, R)).astype(np.float32)
        got = pasta.pasta_rows_times(torch.from_numpy(U).cuda(), torch.from_numpy(W).cuda()).cpu().numpy()
        want = U64 @ W.astype(np.float64)
        # fp32 dot products of R terms: |got - want| <= gamma_R |U| |W|
        assert np.all(np.abs(got - want) <= gamma(R) * (np.abs(U64) @ np.abs(W.astype(np.float64)))), R


def test_fused_update_blocks(env):
    """pasta_cpals_prepare (fp64 R x R algebra) against the exact fp64 chain of the GPU's own GM
    and grams -- W = V^-1, GU = W^T GM W, lambda = sqrt(diag GU), Wn = W / lambda, Gn = GU ./
    lambda lambda^T -- within inverse_error; pasta_rows_times against M Wn (GPU's Wn) within
    gamma_R |M| |Wn| (R#33)."""
    pasta, oracle, torch = env
    rng = np.random.default_rng(1)
    for R in (1, 7, 16, 32, 64):
        grams = [pasta.pasta_gram(torch.from_numpy(rng.uniform(0, 1, (400, R)).astype(np.float32)).cuda())
                 for _ in range(2)]
        M = rng.uniform(-1, 1, size=(3000, R)).astype(np.float32)
        Md = torch.from_numpy(M).cuda()
        GM = pasta.pasta_gram(Md)
        Wn, Gn, lam = pasta.pasta_cpals_prepare(GM, grams)
        GMh = GM.cpu().numpy()
        V = grams[0].cpu().numpy() * grams[1].cpu().numpy()
        dW, W = inverse_error(V)
        nW, nGM = np.linalg.norm(W, 2), np.linalg.norm(GMh, 2)
        GU = W.T @ GMh @ W
        lref = np.sqrt(np.diag(GU))
        # d(GU) <= 2 ||dW|| ||GM|| ||W||  ->  d(lambda_r) <= d(GU_rr) / (2 lambda_r)
        dGU = 2 * dW * nGM * nW + 8 * R * U64E * nW * nW * nGM
        dl = dGU / (2 * lref)
        got_l = lam.cpu().numpy()
        assert np.all(np.abs(got_l - lref) <= 2 * dl + 4 * U64E * lref), (R, got_l, lref)
        Wn_ref = W / lref
        dWn = (dW + nW * dl / lref) / lref  # first order in dW and d(lambda)
        got_W = Wn.cpu().numpy().astype(np.float64)
        assert np.all(np.abs(got_W - Wn_ref) <= U32 * np.abs(Wn_ref) + 2 * dWn[None, :]), R
        Gn_ref = GU / np.outer(lref, lref)
        dGn = (dGU + 2 * np.abs(GU) * (dl / lref)[:, None]) / np.outer(lref, lref)
        assert np.all(np.abs(Gn.cpu().numpy() - Gn_ref) <= 2 * dGn + 4 * U64E * np.abs(Gn_ref)), R
        # apply stage: U = M Wn with the GPU's Wn, fp32 R-term dot products
        U = pasta.pasta_rows_times(Md, Wn).cpu().numpy().astype(np.float64)
        M64 = M.astype(np.float64)
        assert np.all(np.abs(U - M64 @ got_W) <= gamma(R) * (np.abs(M64) @ np.abs(got_W)) + 1e-300), R


def _rounding_perturbation(dims, inds, R, seed):
    """perturb hook for oracle.cpals.cp_als: every stage's result moved by its fp32 rounding
    bound with random signs (R#33): M by gamma_(N + m_i) * sum|terms| (row i holds m_i
    nonzeros: N - 1 products and at most m_i sequential additions per term), each gram by
    gamma_64 |U|^T |U|, the solved factor by one fp32 rounding plus the inverse bound."""
    rng = np.random.default_rng(seed)
    N = len(dims)
    counts = [np.bincount(inds[n], minlength=dims[n]) for n in range(N)]

    def hook(stage, n, pair):
        a, aux = pair
        sign = rng.choice([-1.0, 1.0], size=a.shape)
        if stage == "M":
            g = np.array([gamma(N + int(m)) for m in counts[n]])[:, None]
            return a + sign * g * aux
        if stage == "G":
            return a + sign * gamma(64) * aux
        return a + sign * (U32 + 1e-12) * np.abs(a)
    return hook


@pytest.mark.parametrize("fused", ["1", "0"])
@pytest.mark.parametrize("dims,nnz,R,iters", [((60, 50, 40), 8000, 8, 1), ((60, 50, 40), 8000, 8, 3),
                                               ((40, 30, 20, 10), 6000, 16, 2)])
def test_cpals_matches_oracle(env, dims, nnz, R, iters, fused, monkeypatch):
    """The GPU driver against the fp64 oracle from the same initial factors.  Tolerance =
    4 x the largest deviation of the oracle's own trajectory when every stage is perturbed by
    its fp32 rounding bound (4 seeds) -- the algorithm's sensitivity, computed from the oracle
    alone (R#33), not a number fitted to the kernel."""
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_CPALS_FUSED", fused)
    from oracle.cpals import cp_als
    inds, vals = si.powerlaw_coo(dims, nnz, seed=nnz + R)
    U0 = si.factors(dims, R, seed=R)
    Uo, lam_o, fits_o = cp_als(dims, inds, vals, U0, iters=iters)
    dfit, dlam, dU = 0.0, 0.0, [0.0] * len(dims)
    for sd in range(4):
        Up, lam_p, fits_p = cp_als(dims, inds, vals, U0, iters=iters,
                                   perturb=_rounding_perturbation(dims, inds, R, sd))
        dfit = max(dfit, np.max(np.abs(np.array(fits_p) - fits_o)))
        dlam = max(dlam, np.max(np.abs(lam_p - lam_o) / lam_o))
        dU = [max(d, np.abs(up.astype(np.float64) - uo).max()) for d, up, uo in zip(dU, Up, Uo)]
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    Ud = [torch.from_numpy(u.copy()).cuda() for u in U0]
    lam, fits, it = pasta.pasta_cpals_coo(x, Ud, max_iters=iters, tol=0.0)
    assert it == iters
    assert np.all(np.abs(np.array(fits) - fits_o) <= 4 * dfit + 1e-12), (fits, fits_o, dfit)
    assert np.all(np.abs(lam - lam_o) <= (4 * dlam + 1e-12) * lam_o), (lam, lam_o, dlam)
    for k in range(len(dims)):
        g = Ud[k].cpu().numpy().astype(np.float64)
        assert np.abs(g - Uo[k]).max() <= 4 * dU[k] + 1e-12, (k, np.abs(g - Uo[k]).max(), dU[k])


def test_cpals_recovers_low_rank(env):
    """Exact rank-4 tensor: the fit reaches 0.995, and the residual of the GPU's iterates --
    computed densely in fp64 by the test from the returned factors after every sweep -- never
    increases by more than the resolution of fp32-stored factors, 2 gamma_(N+R+1) ||sum_r
    |lambda_r| |a_r| o |b_r| o |c_r| ||_F (R#33).  (ALS is monotone in exact arithmetic; the
    driver's own fit, ||X||^2 + ||Xhat||^2 - 2 <X, Xhat>, cancels near fit = 1, so it is not
    the quantity checked.)"""
    pasta, oracle, torch = env
    rng = np.random.default_rng(3)
    dims, R = (30, 25, 20), 4
    A = [rng.uniform(0.2, 1.0, size=(d, R)) for d in dims]
    X = np.einsum("ir,jr,kr->ijk", *A)
    inds = np.array(list(itertools.product(*[range(d) for d in dims])), dtype=np.uint32).T
    vals = X[tuple(inds)].astype(np.float32)
    X32 = np.zeros(dims)
    X32[tuple(inds)] = vals
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    Ud = [torch.from_numpy(u).cuda() for u in si.factors(dims, R, seed=9)]
    prev, fits = None, []
    N = len(dims)
    for sweep in range(150):
        lam, f, _ = pasta.pasta_cpals_coo(x, Ud, max_iters=1, tol=0.0)
        fits += f
        U = [u.cpu().numpy().astype(np.float64) for u in Ud]
        Xh = np.einsum("r,ir,jr,kr->ijk", lam, *U)
        Xabs = np.einsum("r,ir,jr,kr->ijk", np.abs(lam), *[np.abs(u) for u in U])
        resid = np.linalg.norm(X32 - Xh)
        slack = 2 * gamma(N + R + 1) * np.linalg.norm(Xabs)
        if prev is not None:
            assert resid <= prev + slack, (sweep, resid, prev, slack)
        prev = resid
    assert fits[-1] > 0.995, fits[-3:]


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
