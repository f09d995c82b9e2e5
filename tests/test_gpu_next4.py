"""GPU parity for SURVEY NEXT-4 through the C ABI: the slice power-law generator (kind 2,
R#30) bit-exact against the oracle's independent generator, and TEW / TS
bit-exact against the oracle (IEEE fp32 results are unique)."""
import numpy as np
import pytest

import synth_inputs as si

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env(oracle_mod):
    import torch

    import paper_conf_iiswc_lilwlob20_b200 as pasta
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    torch.cuda.set_device(0)
    return pasta, oracle_mod, torch


def _export(pasta, x):
    return pasta.pasta_coo_export(x)


def _bits_equal(got, ref):
    got = np.asarray(got, np.float32)
    ref = np.asarray(ref, np.float32)
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(got), nan)
    np.testing.assert_array_equal(got.view(np.uint32)[~nan], ref.view(np.uint32)[~nan])


@pytest.mark.parametrize("dims,nnz,alpha,seed", [
    ((32768, 32768, 76), 50_000, 1.0, 1004),          # irrS-shaped (Table II s4)
    ((1 << 16, 1 << 16, 82, 30), 40_000, 1.0, 1010),  # 4th order, two dense modes
    ((500, 400, 30), 30_000, 0.6, 7),                 # many repeats -> top-up rounds
    ((4, 5, 3), 60, 1.0, 1),                          # saturated box
    ((100000, 20), 2_000, 1.5, 3),                    # N = 2, heavy head
])
def test_slice_powerlaw_generator_bit_exact(env, dims, nnz, alpha, seed):
    pasta, oracle, torch = env
    x = pasta.pasta_gen_powerlaw(dims, nnz, seed, kind=2, alpha=alpha)
    gi, gv = _export(pasta, x)
    oi, ov = oracle.gen_slice_powerlaw(dims, nnz, seed, alpha=alpha)
    np.testing.assert_array_equal(gi, oi)
    np.testing.assert_array_equal(gv.view(np.uint32), ov.view(np.uint32))


@pytest.mark.parametrize("op", ["add", "sub", "mul", "div"])
@pytest.mark.parametrize("n,offset", [(1_000_003, 0), (4096, 1), (7, 0), (0, 0)])
def test_ts_and_tew_values(env, op, n, offset):
    pasta, oracle, torch = env
    rng = np.random.default_rng(n + offset)
    a = rng.uniform(-1, 1, n + offset).astype(np.float32)
    b = rng.uniform(-1, 1, n + offset).astype(np.float32)
    if n >= 8:
        a[offset:offset + 6] = [0.0, -0.0, np.inf, 1e-40, -3e38, 1.0]
    ad = torch.from_numpy(a).cuda()[offset:]  # offset 1: not 16-byte aligned -> scalar path
    bd = torch.from_numpy(b).cuda()[offset:]
    s = np.float32(-0.3125)
    _bits_equal(pasta.pasta_ts(ad, op, s).cpu().numpy(), oracle.ts(a[offset:], op, s))
    _bits_equal(pasta.pasta_tew(ad, bd, op).cpu().numpy(), oracle.tew_same(a[offset:], b[offset:], op))


@pytest.mark.parametrize("op", ["add", "sub", "mul", "div"])
def test_tensor_level_same_and_merged_patterns(env, op):
    pasta, oracle, torch = env
    dims = (3000, 2000, 500)
    xi, xv = si.powerlaw_coo(dims, 200_000, seed=11)
    yi, yv = si.powerlaw_coo(dims, 150_000, seed=12)
    yv[yv == 0] = 0.5
    x = pasta.pasta_coo_from_arrays(dims, xi, xv)
    y = pasta.pasta_coo_from_arrays(dims, yi, yv)
    # TS keeps X's pattern and order
    t = pasta.pasta_coo_ts(x, op, 1.5)
    ti, tv = pasta.pasta_coo_export(t)
    np.testing.assert_array_equal(ti, xi)
    _bits_equal(tv, oracle.ts(xv, op, np.float32(1.5)))
    # same pattern: elementwise in X's order
    x2v = yv[: xi.shape[1]] if yv.shape[0] >= xi.shape[1] else np.resize(yv, xi.shape[1])
    x2 = pasta.pasta_coo_from_arrays(dims, xi, x2v)
    z = pasta.pasta_coo_tew(x, x2, op)
    zi, zv = pasta.pasta_coo_export(z)
    np.testing.assert_array_equal(zi, xi)
    _bits_equal(zv, oracle.tew_same(xv, x2v, op))
    # different patterns: merged, lexicographic
    z = pasta.pasta_coo_tew(x, y, op)
    zi, zv = pasta.pasta_coo_export(z)
    oi, ov = oracle.tew_merge(xi, xv, yi, yv, op)
    np.testing.assert_array_equal(zi, oi)
    _bits_equal(zv, ov)


def test_tew_errors(env):
    pasta, oracle, torch = env
    x = pasta.pasta_coo_from_arrays((5, 5), np.array([[0, 0], [1, 1]], np.uint32), np.ones(2, np.float32))
    y = pasta.pasta_coo_from_arrays((5, 5), np.array([[2], [3]], np.uint32), np.ones(1, np.float32))
    with pytest.raises(pasta.PastaError):
        pasta.pasta_coo_tew(x, y, "add")  # repeated coordinate inside x
    w = pasta.pasta_coo_from_arrays((5, 6), np.array([[2], [3]], np.uint32), np.ones(1, np.float32))
    with pytest.raises(pasta.PastaError):
        pasta.pasta_coo_tew(y, w, "add")  # shapes differ
