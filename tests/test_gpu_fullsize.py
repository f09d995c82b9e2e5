"""Full-size parity (BASELINE.json sizes, the launch configuration bench.py times) on
sampled outputs: 4096 random rows + the 64 heaviest rows of every mode, checked against the
oracle computed row by row on the same host arrays.  Plus a full-size generator pin: the
oracle's independently generated first-200k-distinct nonzeros of the bench workload's draw
sequence must appear, with identical values, in the GPU generator's 100M-nonzero tensor."""
import numpy as np
import pytest

import synth_inputs as si

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.fixture(scope="module")
def env(oracle_mod):
    import torch

    import paper_conf_iiswc_lilwlob20_b200 as pasta
    assert torch.cuda.is_available()
    torch.cuda.set_device(0)
    return pasta, oracle_mod, torch


def _sample_rows(inds_n, dim, rng):
    heavy = np.argsort(np.bincount(inds_n, minlength=dim))[-64:]
    rnd = rng.integers(0, dim, size=4096)
    return np.unique(np.concatenate([heavy, rnd]).astype(np.uint32))


@pytest.mark.parametrize("key", ["h", "c4", "c2", "c3"])
def test_fullsize_sampled_rows(env, key):
    pasta, oracle, torch = env
    cfg = si.CONFIGS[key]
    dims, R, M = cfg["dims"], cfg["R"], cfg["nnz"]
    inds, vals = si.powerlaw_coo(dims, M, seed=cfg["seed"] + 77, dedup=False)
    g = torch.Generator(device="cuda")
    g.manual_seed(5)
    Ud = [torch.rand((d, R), generator=g, device="cuda") for d in dims]
    U = [u.cpu().numpy() for u in Ud]
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_coo_to_hicoo(x, 7)
    rng = np.random.default_rng(1)
    for n in range(len(dims)):
        rows = _sample_rows(inds[n], dims[n], rng)
        ref, ab = oracle.mttkrp_rows(dims, inds, vals, n, U, rows)
        for name, fn, t in (("coo", pasta.pasta_mttkrp_coo, x), ("hicoo", pasta.pasta_mttkrp_hicoo, h)):
            got = fn(t, n, Ud)[torch.from_numpy(rows.astype(np.int64)).cuda()].cpu().numpy()
            excess = np.abs(got.astype(np.float64) - ref) - (1e-4 * ab + 1e-6)
            assert excess.max() <= 0, f"{key} {name} mode {n}: excess {excess.max():.3e}"
        del ref, ab


def test_fullsize_generator_contains_oracle_prefix(env):
    pasta, oracle, torch = env
    cfg = si.CONFIGS["h"]
    dims, M = cfg["dims"], cfg["nnz"]
    x = pasta.pasta_gen_powerlaw(dims, M, cfg["seed"])
    gi, gv = pasta.pasta_coo_export(x)
    assert gi.shape == (3, M)
    # lexicographically sorted, unique, in range
    d0 = np.diff(gi[0].astype(np.int64))
    assert np.all(d0 >= 0)
    same0 = d0 == 0
    d1 = np.diff(gi[1].astype(np.int64))
    assert np.all(d1[same0] >= 0)
    same01 = same0 & (d1 == 0)
    assert np.all(np.diff(gi[2].astype(np.int64))[same01] > 0)
    for k in range(3):
        assert gi[k].max() < dims[k]
    oi, ov = oracle.gen_powerlaw(dims, 200_000, cfg["seed"])
    # membership of every oracle coordinate (with its value) in the sorted GPU output
    lo = np.searchsorted(gi[0], oi[0], side="left")
    hi = np.searchsorted(gi[0], oi[0], side="right")
    found = 0
    for j in range(oi.shape[1]):
        a, b = lo[j], hi[j]
        a1 = a + np.searchsorted(gi[1][a:b], oi[1, j], side="left")
        b1 = a + np.searchsorted(gi[1][a:b], oi[1, j], side="right")
        p = a1 + np.searchsorted(gi[2][a1:b1], oi[2, j], side="left")
        assert p < b1 and gi[2][p] == oi[2, j], f"oracle nonzero {j} missing"
        assert gv[p].view(np.uint32) == ov[j].view(np.uint32)
        found += 1
    assert found == 200_000


def test_fullsize_hicoo_conversion_and_mode_sort_bit_exact(env):
    """Integer work at a BASELINE.json size (C4: 54M nonzeros, 4th order): the GPU COO->HiCOO
    conversion (B = 128) and the mode-3 sort equal the oracle's qsort-based ones bit for bit."""
    pasta, oracle, torch = env
    cfg = si.CONFIGS["c4"]
    dims, M = cfg["dims"], cfg["nnz"]
    inds, vals = si.powerlaw_coo(dims, M, seed=cfg["seed"] + 5, dedup=False)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_hicoo_export(pasta.pasta_coo_to_hicoo(x, 7))
    o = oracle.coo_to_hicoo(inds, vals, 7)
    assert h["nblocks"] == o["nblocks"]
    for key in ("bptr", "binds", "einds"):
        assert np.array_equal(h[key], o[key]), key
    assert np.array_equal(h["vals"].view(np.uint32), o["vals"].view(np.uint32))
    del h, o
    gi, gv = pasta.pasta_coo_export_mode(x, 3)
    oi, ov = oracle.mode_sort(inds, vals, 3)
    assert np.array_equal(gi, oi) and np.array_equal(gv.view(np.uint32), ov.view(np.uint32))


@pytest.mark.parametrize("key", ["h", "c3"])
def test_fullsize_ghicoo_sampled_rows(env, key):
    """gHiCOO (NEXT-2) with the storage-minimising mask, as bench.py times it, at full size."""
    pasta, oracle, torch = env
    cfg = si.CONFIGS[key]
    dims, R, M = cfg["dims"], cfg["R"], cfg["nnz"]
    inds, vals = si.powerlaw_coo(dims, M, seed=cfg["seed"] + 91, dedup=False)
    g = torch.Generator(device="cuda")
    g.manual_seed(7)
    Ud = [torch.rand((d, R), generator=g, device="cuda") for d in dims]
    U = [u.cpu().numpy() for u in Ud]
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    gh = pasta.pasta_coo_to_ghicoo(x, 7, 0)
    assert 0 < gh.cmask < (1 << len(dims))
    rng = np.random.default_rng(2)
    for n in range(len(dims)):
        rows = _sample_rows(inds[n], dims[n], rng)
        ref, ab = oracle.mttkrp_rows(dims, inds, vals, n, U, rows)
        got = pasta.pasta_mttkrp_hicoo(gh, n, Ud)[torch.from_numpy(rows.astype(np.int64)).cuda()].cpu().numpy()
        excess = np.abs(got.astype(np.float64) - ref) - (1e-4 * ab + 1e-6)
        assert excess.max() <= 0, f"{key} ghicoo mask {gh.cmask:b} mode {n}: excess {excess.max():.3e}"
        del ref, ab


def test_fullsize_ghicoo_conversion_bit_exact(env):
    pasta, oracle, torch = env
    cfg = si.CONFIGS["c4"]
    dims, M = cfg["dims"], cfg["nnz"]
    inds, vals = si.powerlaw_coo(dims, M, seed=cfg["seed"] + 6, dedup=False)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    mask = 0b0101
    gx = pasta.pasta_ghicoo_export(pasta.pasta_coo_to_ghicoo(x, 7, mask))
    o = oracle.coo_to_ghicoo(inds, vals, 7, mask)
    assert gx["nblocks"] == o["nblocks"]
    assert np.array_equal(gx["bptr"], o["bptr"])
    for k in range(4):
        for key in ("binds", "einds", "uinds"):
            if o[key][k] is not None:
                assert np.array_equal(gx[key][k], o[key][k]), (key, k)
    assert np.array_equal(gx["vals"].view(np.uint32), o["vals"].view(np.uint32))


def test_fullsize_ts_tew_bit_exact(env):
    """TEW / TS (NEXT-4) on the bench's 100M-element value arrays, every element."""
    pasta, oracle, torch = env
    M = si.CONFIGS["h"]["nnz"]
    rng = np.random.default_rng(3)
    a = rng.uniform(-1, 1, M).astype(np.float32)
    b = rng.uniform(-1, 1, M).astype(np.float32)
    ad, bd = torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda()
    for op in ("mul", "div"):
        got = pasta.pasta_ts(ad, op, 0.5).cpu().numpy()
        assert np.array_equal(got.view(np.uint32), oracle.ts(a, op, np.float32(0.5)).view(np.uint32)), op
    for op in ("add", "sub"):
        got = pasta.pasta_tew(ad, bd, op).cpu().numpy()
        assert np.array_equal(got.view(np.uint32), oracle.tew_same(a, b, op).view(np.uint32)), op


def test_fullsize_slice_powerlaw_contains_oracle_prefix(env):
    """irrL-shaped (Table II s6: (4.2M)^2 x 168, 84M nonzeros) slice power-law tensor on the GPU
    contains the oracle's independently generated first 200k distinct nonzeros, same values."""
    pasta, oracle, torch = env
    dims, M, seed = (4_200_000, 4_200_000, 168), 84_000_000, 1006
    x = pasta.pasta_gen_powerlaw(dims, M, seed, kind=2)
    gi, gv = pasta.pasta_coo_export(x)
    assert gi.shape == (3, M)
    oi, ov = oracle.gen_slice_powerlaw(dims, 200_000, seed)
    key_g = (gi[0].astype(np.uint64) << np.uint64(40)) | (gi[1].astype(np.uint64) << np.uint64(8)) \
        | gi[2].astype(np.uint64)
    key_o = (oi[0].astype(np.uint64) << np.uint64(40)) | (oi[1].astype(np.uint64) << np.uint64(8)) \
        | oi[2].astype(np.uint64)
    assert np.all(key_g[1:] > key_g[:-1])  # lexicographic, distinct
    pos = np.searchsorted(key_g, key_o)
    assert np.all(pos < M) and np.array_equal(key_g[pos], key_o)
    assert np.array_equal(gv[pos].view(np.uint32), ov.view(np.uint32))


def test_fullsize_c5_one_billion_mode0(env):
    """BASELINE config 5 (regL-shaped, 1B nonzeros, R = 32): mode-0 MTTKRP on sampled rows
    against the oracle.  The input is drawn on the host by synth_inputs (same product-form law
    as the GPU generator, no dedup), never exported from the CUDA path.  Needs ~40 GB of host
    memory; skipped when the host has less than 96 GB available."""
    import psutil
    if psutil.virtual_memory().available < 96 * (1 << 30):
        pytest.skip("needs >= 96 GB of available host memory")
    pasta, oracle, torch = env
    cfg = si.CONFIGS["c5"]
    dims, R, M = cfg["dims"], cfg["R"], cfg["nnz"]
    inds, vals = si.powerlaw_coo_lean(dims, M, seed=cfg["seed"] + 3)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    g = torch.Generator(device="cuda")
    g.manual_seed(11)
    Ud = [torch.rand((d, R), generator=g, device="cuda") for d in dims]
    rows = _sample_rows(inds[0], dims[0], np.random.default_rng(4))[:1024]
    got = pasta.pasta_mttkrp_coo(x, 0, Ud)[torch.from_numpy(rows.astype(np.int64)).cuda()].cpu().numpy()
    del x
    U = [u.cpu().numpy() for u in Ud]
    ref, ab = oracle.mttkrp_rows(dims, inds, vals, 0, U, rows)
    excess = np.abs(got.astype(np.float64) - ref) - (1e-4 * ab + 1e-6)
    assert excess.max() <= 0, f"c5 mode 0: excess {excess.max():.3e}"
