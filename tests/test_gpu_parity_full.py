"""Parity at the edges of the north_star tolerance and at full size (SURVEY 8(c) "GPU tolerance"
row; P:157 / P:282 atomics; P:181 / P:205-207 HiCOO).

* A single output row holding 10^7 nonzeros, in each mode in turn, every mode of COO and HiCOO
  MTTKRP checked element by element: the case where a flat sequential fp32 sum would fail
  (~1.1e-4 relative over 10^7 terms) and only hierarchical summation
  (register runs + vector atomics at run ends) stays within 1e-4 * sum|terms| + 1e-6.
* The headline workload H (regL-shaped (2^23)^3, 100M nonzeros, R = 16, the launch
  configuration bench.py times): EVERY output row of every mode, COO and HiCOO, against the full
  oracle.
* COO -> HiCOO (B = 128) bit-exact (memcmp of bptr / binds / einds / vals) at the full sizes of
  H, C2 and C3 (C4 is in test_gpu_fullsize.py).
Inputs come from synth_inputs only, never from the CUDA path.
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
    assert torch.cuda.is_available()
    torch.cuda.set_device(0)
    return pasta, oracle_mod, torch


def _excess(got, ref, ab):
    g = got.detach().cpu().numpy().astype(np.float64)
    return np.abs(g - ref) - (TOL_REL * ab + TOL_ABS)


@pytest.mark.parametrize("force_hot", ["0", "1"])
@pytest.mark.parametrize("hot_mode", [0, 1, 2])
def test_hot_row_ten_million(env, hot_mode, force_hot, monkeypatch):
    """10^7 nonzeros in row 1234 of mode `hot_mode` (+ 10^6 uniform elsewhere), R = 16.  With
    force_hot = 1 the hot-row cache tiers are on, so when the hot mode is a gathered mode its
    row is served from the shared-memory tier."""
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_HOT_FORCE", force_hot)
    dims = (4096, 4096, 4096)
    inds, vals = si.hot_row_coo(dims, 10_000_000, 1_000_000, seed=31 + hot_mode, mode=hot_mode, hot_row=1234)
    assert np.count_nonzero(inds[hot_mode] == 1234) == 10_000_000
    U = si.factors(dims, 16, seed=7)
    Ud = [torch.from_numpy(u).cuda() for u in U]
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_coo_to_hicoo(x, 7)
    for n in range(3):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        for name, got in (("coo", pasta.pasta_mttkrp_coo(x, n, Ud)), ("hicoo", pasta.pasta_mttkrp_hicoo(h, n, Ud))):
            ex = _excess(got, ref, ab)
            assert ex.max() <= 0, f"{name} hot mode {hot_mode} mode {n}: excess {ex.max():.3e}"
            if n == hot_mode:  # the 10^7-term row itself: report how far inside the bound it is
                g = got[1234].cpu().numpy().astype(np.float64)
                rel = np.max(np.abs(g - ref[1234]) / ab[1234])
                assert rel < TOL_REL, (name, rel)


def test_fullsize_h_every_row(env):
    """H at full size: every row of every mode, COO and HiCOO, vs the full fp64 oracle."""
    pasta, oracle, torch = env
    cfg = si.CONFIGS["h"]
    dims, R, M = cfg["dims"], cfg["R"], cfg["nnz"]
    inds, vals = si.powerlaw_coo_lean(dims, M, seed=cfg["seed"] + 101)
    g = torch.Generator(device="cuda")
    g.manual_seed(13)
    Ud = [torch.rand((d, R), generator=g, device="cuda") for d in dims]
    U = [u.cpu().numpy() for u in Ud]
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_coo_to_hicoo(x, 7)
    for n in range(3):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        for name, fn, t in (("coo", pasta.pasta_mttkrp_coo, x), ("hicoo", pasta.pasta_mttkrp_hicoo, h)):
            ex = _excess(fn(t, n, Ud), ref, ab)
            assert ex.max() <= 0, f"h {name} mode {n}: excess {ex.max():.3e} at row {np.argmax(ex) // R}"
            del ex
        del ref, ab


@pytest.mark.parametrize("key", ["h", "c2", "c3"])
def test_fullsize_hicoo_conversion_bit_exact(env, key):
    pasta, oracle, torch = env
    cfg = si.CONFIGS[key]
    dims, M = cfg["dims"], cfg["nnz"]
    if key == "h":
        inds, vals = si.powerlaw_coo_lean(dims, M, seed=cfg["seed"] + 5)
    else:
        inds, vals = si.powerlaw_coo(dims, M, seed=cfg["seed"] + 5, dedup=False)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    hx = pasta.pasta_hicoo_export(pasta.pasta_coo_to_hicoo(x, 7))
    del x
    o = oracle.coo_to_hicoo(inds, vals, 7)
    assert hx["nblocks"] == o["nblocks"]
    for k in ("bptr", "binds", "einds"):
        assert np.array_equal(hx[k], o[k]), k
    assert np.array_equal(hx["vals"].view(np.uint32), o["vals"].view(np.uint32))


@pytest.mark.parametrize("tier", ["1", "2"])
@pytest.mark.parametrize("hot_mb", ["0.05", "64"])
def test_hicoo_hot_block_tiers_retag(env, hot_mb, tier, monkeypatch):
    """HiCOO hot-row tiers, shared-memory and L2 tiers forced on: tier = 1 hot-block tiers (R#34,
    retagged canonical blocks), tier = 2 tier blocks (R#36, the copy rebuilt over heat-ranked
    blocks).  Ragged dims (partial last blocks), and the rank changed on the same handle (R = 16
    -> 32 -> 8 -> 16) so the tiers are rebuilt between launches; every result against the
    oracle.  hot_mb = 0.05 leaves most rows cold (mixed tags inside a warp's window)."""
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_HICOO_HOT", tier)
    monkeypatch.setenv("PASTA_HOT_FORCE", "1")
    monkeypatch.setenv("PASTA_HOT_MB", hot_mb)
    dims = (1000, 777, 1300)
    inds, vals = si.powerlaw_coo(dims, 300_000, seed=77)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_coo_to_hicoo(x, 7)
    gh = pasta.pasta_coo_to_ghicoo(x, 7, 0b101)  # mode 1 uncompressed: tiers on modes 0 and 2 only
    for R in (16, 32, 8, 16):
        U = si.factors(dims, R, seed=R)
        Ud = [torch.from_numpy(u).cuda() for u in U]
        for n in range(3):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
            for name, t in (("hicoo", h), ("ghicoo", gh)):
                ex = _excess(pasta.pasta_mttkrp_hicoo(t, n, Ud), ref, ab)
                assert ex.max() <= 0, f"{name} R={R} mode {n}: excess {ex.max():.3e}"


def test_hicoo_tier_blocks_switch(env, monkeypatch):
    """R#36 tier blocks on one handle while the tier mode flips (2 -> 0 -> 1 -> 2 -> generic
    R = 12 path -> 2): the copy is rebuilt plain / tiered / retagged each time and every result
    matches the oracle; order 4 with a gHiCOO mask; the canonical HiCOO arrays never change."""
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_HOT_FORCE", "1")
    monkeypatch.setenv("PASTA_HOT_MB", "0.1")
    dims = (300, 520, 41, 700)
    inds, vals = si.powerlaw_coo(dims, 200_000, seed=91)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_coo_to_hicoo(x, 7)
    gh = pasta.pasta_coo_to_ghicoo(x, 7, 0b1011)  # mode 2 uncompressed
    before = pasta.pasta_hicoo_export(h)
    for tier, R in (("2", 16), ("0", 16), ("1", 16), ("2", 32), ("2", 64), ("2", 12), ("2", 16)):
        monkeypatch.setenv("PASTA_HICOO_HOT", tier)
        U = si.factors(dims, R, seed=R + 3)
        Ud = [torch.from_numpy(u).cuda() for u in U]
        for n in range(4):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
            for name, t in (("hicoo", h), ("ghicoo", gh)):
                ex = _excess(pasta.pasta_mttkrp_hicoo(t, n, Ud), ref, ab)
                assert ex.max() <= 0, f"{name} tier {tier} R={R} mode {n}: excess {ex.max():.3e}"
    after = pasta.pasta_hicoo_export(h)
    for k in ("bptr", "binds", "einds"):
        assert np.array_equal(before[k], after[k]), k
    assert np.array_equal(before["vals"].view(np.uint32), after["vals"].view(np.uint32))


@pytest.mark.parametrize("hot,cfg", [("0", "0"), ("2", "0"), ("2", "2"), ("2", "3")])
def test_hicoo_staged_orders_ranks(env, hot, cfg, monkeypatch):
    """The staged HiCOO kernels (plain decode WA 9, tier blocks WA 10 / 17) in every shape
    (PASTA_HS_CFG 0 = 16 warps x 4-nonzero steps, 2 = 16 x 8, 3 = 12 x 8) at orders 2, 3, 4 and
    R = 16, 32, 64, tiers forced on (order 2 at R >= 32 once faulted with cache-hinted decode
    loads; the decode now uses ld.cs)."""
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_HICOO_HOT", hot)
    monkeypatch.setenv("PASTA_HS_CFG", cfg)
    monkeypatch.setenv("PASTA_HOT_FORCE", "1")
    monkeypatch.setenv("PASTA_HOT_MB", "0.2")
    for dims in ((5000, 3000), (900, 1300, 700), (300, 520, 41, 700)):
        inds, vals = si.powerlaw_coo(dims, 120_000, seed=5)
        x = pasta.pasta_coo_from_arrays(dims, inds, vals)
        h = pasta.pasta_coo_to_hicoo(x, 7)
        for R in (16, 32, 64):
            U = si.factors(dims, R, seed=R + 11)
            Ud = [torch.from_numpy(u).cuda() for u in U]
            for n in range(len(dims)):
                ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
                ex = _excess(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab)
                assert ex.max() <= 0, f"hot {hot} cfg {cfg} dims {dims} R={R} mode {n}: excess {ex.max():.3e}"
                if R == 32:  # two row shards (pasta_hicoo_shard) into one output, tiers rebuilt per shard
                    b = pasta.pasta_coo_partition(x, n, 2)
                    out = torch.zeros((dims[n], R), device="cuda")
                    for q in range(2):
                        pasta.pasta_mttkrp_hicoo(pasta.pasta_hicoo_shard(h, n, int(b[q]), int(b[q + 1])), n, Ud, out=out)
                    ex = _excess(out, ref, ab)
                    assert ex.max() <= 0, f"shards hot {hot} cfg {cfg} dims {dims} mode {n}: excess {ex.max():.3e}"


@pytest.mark.parametrize("shape", ["12x8", "16x4"])
def test_hicoo_tier_blocks_orders_2_3(env, shape, monkeypatch):
    """R#36 tier blocks with both tiers forced on, at orders 2 (SpMM-like) and 3, in the default
    12-warp x 8-nonzero-step shape and the 16 x 4 shape, R = 16 and 32."""
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_HICOO_HOT", "2")
    monkeypatch.setenv("PASTA_HOT_FORCE", "1")
    monkeypatch.setenv("PASTA_HOT_MB", "0.2")
    monkeypatch.setenv("PASTA_HS_CFG", "3" if shape == "12x8" else "0")
    for dims, nnz, seed in (((5000, 3000), 120_000, 5), ((900, 1300, 700), 250_000, 6)):
        inds, vals = si.powerlaw_coo(dims, nnz, seed=seed)
        x = pasta.pasta_coo_from_arrays(dims, inds, vals)
        h = pasta.pasta_coo_to_hicoo(x, 7)
        for R in (16, 32):
            U = si.factors(dims, R, seed=R + 11)
            Ud = [torch.from_numpy(u).cuda() for u in U]
            for n in range(len(dims)):
                ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
                ex = _excess(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab)
                assert ex.max() <= 0, f"{shape} dims {dims} R={R} mode {n}: excess {ex.max():.3e}"
