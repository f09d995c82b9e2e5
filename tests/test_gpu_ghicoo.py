"""GPU parity of gHiCOO (R#29) through the C ABI.

* conversion: bit-exact against the oracle's conversion for every mask tried;
* MTTKRP on gHiCOO handles: |gpu - ref| <= 1e-4 * sum|terms| + 1e-6 against O-MTTKRP;
* hypersparse-aware mask choice: the GPU's choice equals the argmin, over every non-empty
  mask, of the storage formula evaluated with the oracle's block counts.
"""
import numpy as np
import pytest

import synth_inputs as si

pytestmark = pytest.mark.gpu

TOL_REL, TOL_ABS = 1e-4, 1e-6


@pytest.fixture(scope="module")
def env(oracle_mod):
    import torch

    import paper_conf_iiswc_lilwlob20_b200 as pasta
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    torch.cuda.set_device(0)
    return pasta, oracle_mod, torch


def _check(got, ref, ab, what=""):
    g = got.detach().cpu().numpy().astype(np.float64)
    excess = np.abs(g - ref) - (TOL_REL * ab + TOL_ABS)
    i = np.unravel_index(np.argmax(excess), excess.shape) if excess.size else None
    assert excess.size == 0 or excess.max() <= 0, (
        f"{what}: tolerance exceeded at {i}: gpu={g[i]!r} ref={ref[i]!r} sumabs={ab[i]!r}")


def _same(g, o):
    assert g["nblocks"] == o["nblocks"]
    np.testing.assert_array_equal(g["bptr"], o["bptr"])
    for k in range(g["order"]):
        for key in ("binds", "einds", "uinds"):
            if o[key][k] is None:
                assert g[key][k] is None
            else:
                np.testing.assert_array_equal(g[key][k], o[key][k], err_msg=f"{key}[{k}]")
    np.testing.assert_array_equal(g["vals"].view(np.uint32), o["vals"].view(np.uint32))


CASES = [
    # dims, nnz, gen, block_bits, masks
    ((300, 200, 500), 40_000, "powerlaw", 7, [0b001, 0b010, 0b100, 0b011, 0b101, 0b110, 0b111]),
    ((320, 28000, 1600), 60_000, "powerlaw", 7, [0b001, 0b101, 0b111]),   # flickr-like shape
    ((60, 70, 80, 90), 30_000, "uniform", 4, [0b0001, 0b1010, 0b0111, 0b1111]),
    ((20, 30, 25, 12, 9), 10_000, "uniform", 3, [0b00100, 0b10011]),     # N = 5
    ((1000, 900), 20_000, "powerlaw", 5, [0b01, 0b10]),                   # N = 2
]


@pytest.mark.parametrize("dims,nnz,gen,bb,masks", CASES)
def test_conversion_bit_exact_and_mttkrp(env, dims, nnz, gen, bb, masks):
    pasta, oracle, torch = env
    mk = si.powerlaw_coo if gen == "powerlaw" else si.uniform_coo
    inds, vals = mk(dims, nnz, seed=nnz + bb)
    U = si.factors(dims, 16, seed=7)
    Ud = [torch.from_numpy(u).cuda() for u in U]
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    refs = [oracle.mttkrp(dims, inds, vals, n, U) for n in range(len(dims))]
    for m in masks:
        g = pasta.pasta_coo_to_ghicoo(x, bb, m)
        assert g.cmask == m
        _same(pasta.pasta_ghicoo_export(g), oracle.coo_to_ghicoo(inds, vals, bb, m))
        for n in range(len(dims)):
            ref, ab = refs[n]
            _check(pasta.pasta_mttkrp_hicoo(g, n, Ud), ref, ab, f"ghicoo {dims} mask {m:b} mode {n}")


def test_full_mask_equals_hicoo_handle(env):
    pasta, oracle, torch = env
    dims = (4096, 4096, 4096)
    inds, vals = si.powerlaw_coo(dims, 100_000, seed=3)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    g = pasta.pasta_ghicoo_export(pasta.pasta_coo_to_ghicoo(x, 7, 0b111))
    h = pasta.pasta_hicoo_export(pasta.pasta_coo_to_hicoo(x, 7))
    np.testing.assert_array_equal(g["bptr"], h["bptr"])
    for k in range(3):
        np.testing.assert_array_equal(g["binds"][k], h["binds"][k])
        np.testing.assert_array_equal(g["einds"][k], h["einds"][k])


@pytest.mark.parametrize("dims,nnz,bb", [((320, 28000, 1600), 50_000, 7),
                                         ((4096, 4096, 4096), 80_000, 7),
                                         ((60, 70, 80, 90), 30_000, 3)])
def test_auto_mask_is_storage_argmin(env, dims, nnz, bb):
    pasta, oracle, torch = env
    inds, vals = si.powerlaw_coo(dims, nnz, seed=21)
    N, M = len(dims), inds.shape[1]
    best, best_b = None, None
    for m in range(1, 1 << N):  # ascending: ties keep the smallest mask
        nb = oracle.coo_to_ghicoo(inds, vals, bb, m)["nblocks"]
        nc = bin(m).count("1")
        b = (nc + 4 * (N - nc) + 4) * M + (8 + 4 * nc) * nb
        if best_b is None or b < best_b:
            best, best_b = m, b
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    cm, nbytes = pasta.pasta_ghicoo_auto_mask(x, bb)
    assert (cm, nbytes) == (best, best_b)
    g = pasta.pasta_coo_to_ghicoo(x, bb, 0)
    assert g.cmask == best


def test_empty_and_invalid(env):
    pasta, oracle, torch = env
    x = pasta.pasta_coo_from_arrays((10, 20, 30), np.zeros((3, 0), np.uint32), np.zeros(0, np.float32))
    g = pasta.pasta_coo_to_ghicoo(x, 7, 0b101)
    assert g.nblocks == 0 and g.nnz == 0
    U = [torch.rand(d, 16, device="cuda") for d in (10, 20, 30)]
    out = pasta.pasta_mttkrp_hicoo(g, 1, U)
    assert torch.all(out == 0)
    inds, vals = si.uniform_coo((10, 20, 30), 50, seed=1)
    x = pasta.pasta_coo_from_arrays((10, 20, 30), inds, vals)
    with pytest.raises(pasta.PastaError):
        pasta.pasta_coo_to_ghicoo(x, 7, 0b1000)
    with pytest.raises(pasta.PastaError):
        pasta.pasta_coo_to_ghicoo(x, 9, 0b1)
    g = pasta.pasta_coo_to_ghicoo(x, 7, 0b1)
    with pytest.raises(pasta.PastaError):
        pasta.pasta_hicoo_export(g)
