"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle.

Tolerance (BASELINE.json north_star): |gpu - ref| <= 1e-4 * sum|terms| + 1e-6
per output element.  Integer / byte work (generator, mode sort, HiCOO conversion) is
compared bit for bit.  Inputs come from synth_inputs or from the oracle's own generator,
never from the CUDA path.
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
    g = got.detach().cpu().numpy().astype(np.float64) if hasattr(got, "detach") else got
    excess = np.abs(g - ref) - (TOL_REL * ab + TOL_ABS)
    i = np.unravel_index(np.argmax(excess), excess.shape) if excess.size else None
    assert excess.size == 0 or excess.max() <= 0, (
        f"{what}: tolerance exceeded at {i}: gpu={g[i]!r} ref={ref[i]!r} sumabs={ab[i]!r}")


def _dev(torch, U):
    return [torch.from_numpy(np.ascontiguousarray(u)).cuda() for u in U]


def test_config1_all_modes_coo_and_hicoo(env):
    pasta, oracle, torch = env
    cfg = si.CONFIGS["c1"]
    dims, R = cfg["dims"], cfg["R"]
    inds, vals = si.uniform_coo(dims, cfg["nnz"], seed=cfg["seed"])
    U = si.factors(dims, R, seed=cfg["seed"])
    Ud = _dev(torch, U)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_coo_to_hicoo(x, 7)
    for n in range(3):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        _check(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, f"coo mode {n}")
        _check(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab, f"hicoo mode {n}")


CASES = [
    # dims, nnz, R, generator, block_bits
    ((300, 200, 500), 50_013, 16, "powerlaw", 7),
    ((300, 200, 500), 50_013, 32, "uniform", 7),
    ((1000, 900), 30_001, 16, "powerlaw", 5),          # N = 2 (SpMM)
    ((60, 70, 80, 90), 40_007, 16, "powerlaw", 4),     # N = 4
    ((20, 30, 25, 12, 9), 20_003, 8, "uniform", 3),    # N = 5, generic order path
    ((400, 300, 200), 25_000, 1, "powerlaw", 7),       # R = 1, scalar path
    ((400, 300, 200), 25_000, 3, "uniform", 6),        # R % 4 != 0
    ((400, 300, 200), 25_000, 40, "powerlaw", 7),      # R = 40: 16 lanes, ragged lanes
    ((400, 300, 200), 12_345, 160, "powerlaw", 8),     # R > 128: column loop
    ((1, 500, 300), 20_000, 16, "uniform", 7),         # a dimension of 1
    ((4096, 4096, 4096), 200_000, 16, "powerlaw", 7),  # several tiles, hypersparse blocks
    ((3000, 2000, 4000), 300_000, 8, "powerlaw", 7),   # R = 8: 2 lanes per nonzero
    ((3000, 2000, 4000), 200_000, 64, "powerlaw", 7),  # R = 64: 16 lanes per nonzero
    ((60, 70, 80, 90), 100_000, 64, "powerlaw", 4),    # N = 4, R = 64
    ((2000, 1500), 100_000, 8, "uniform", 6),          # N = 2, R = 8
]


@pytest.mark.parametrize("dims,nnz,R,gen,bb", CASES)
def test_random_tensors_all_modes(env, dims, nnz, R, gen, bb):
    pasta, oracle, torch = env
    seed = nnz + R
    mk = si.powerlaw_coo if gen == "powerlaw" else si.uniform_coo
    inds, vals = mk(dims, nnz, seed=seed)  # shuffled (unsorted) input order
    U = si.factors(dims, R, seed=seed)
    Ud = _dev(torch, U)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_coo_to_hicoo(x, bb)
    for n in range(len(dims)):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        _check(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, f"coo {dims} R={R} mode {n}")
        _check(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab, f"hicoo {dims} R={R} mode {n}")


def test_hot_row_spanning_many_warps(env):
    """2M nonzeros in one output row: the segmented reduction must carry across groups,
    warps and CTAs, and hierarchical summation must stay inside the tolerance."""
    pasta, oracle, torch = env
    dims = (5000, 3000, 2000)
    inds, vals = si.hot_row_coo(dims, 2_000_000, 100_000, seed=3, mode=0, hot_row=1234)
    U = si.factors(dims, 16, seed=5)
    Ud = _dev(torch, U)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_coo_to_hicoo(x, 7)
    for n in range(3):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        _check(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, f"coo hot mode {n}")
        _check(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab, f"hicoo hot mode {n}")


def test_output_is_overwritten_and_empty_rows_zero(env):
    pasta, oracle, torch = env
    dims = (1000, 50, 60)
    inds, vals = si.uniform_coo((1000, 50, 60), 3000, seed=1)
    keep = inds[0] % 3 != 0  # every third row empty
    inds, vals = np.ascontiguousarray(inds[:, keep]), vals[keep]
    U = si.factors(dims, 16, seed=2)
    Ud = _dev(torch, U)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_coo_to_hicoo(x, 7)
    ref, ab = oracle.mttkrp(dims, inds, vals, 0, U)
    for fn, t in ((pasta.pasta_mttkrp_coo, x), (pasta.pasta_mttkrp_hicoo, h)):
        out = torch.full((dims[0], 16), 7.0, device="cuda")
        fn(t, 0, Ud, out=out)
        _check(out, ref, ab, fn.__name__)
        assert torch.all(out[0::3] == 0)


def test_empty_tensor_and_order_one(env):
    pasta, oracle, torch = env
    dims = (10, 20, 30)
    x = pasta.pasta_coo_from_arrays(dims, np.zeros((3, 0), np.uint32), np.zeros(0, np.float32))
    Ud = _dev(torch, si.factors(dims, 16, seed=0))
    out = torch.full((20, 16), 3.0, device="cuda")
    pasta.pasta_mttkrp_coo(x, 1, Ud, out=out)
    assert torch.all(out == 0)
    h = pasta.pasta_coo_to_hicoo(x, 7)
    assert h.nblocks == 0
    out.fill_(3.0)
    pasta.pasta_mttkrp_hicoo(h, 1, Ud, out=out)
    assert torch.all(out == 0)
    # order 1: the empty Khatri-Rao product; MTTKRP = slice sums in every column
    i1 = np.array([[5, 1, 5, 9]], np.uint32)
    v1 = np.array([1.0, 2.0, -0.5, 4.0], np.float32)
    x1 = pasta.pasta_coo_from_arrays((10,), i1, v1)
    got = pasta.pasta_mttkrp_coo(x1, 0, [None], R=4).cpu().numpy()
    ref, ab = oracle.mttkrp((10,), i1, v1, 0, [None], R=4)
    _check(got, ref, ab, "order 1")


def test_generator_bit_exact_with_oracle(env):
    pasta, oracle, torch = env
    cases = [
        dict(dims=(12092, 9184, 28818), nnz=200_000, seed=1002),
        dict(dims=(6066, 5699, 244268, 1176), nnz=100_000, seed=1004),
        dict(dims=(64, 64, 64), nnz=20_000, seed=7),  # many repeated draws
        dict(dims=(1 << 16, 1 << 16), nnz=5000, seed=3, initiator=[0.57, 0.19, 0.19, 0.05]),
        dict(dims=(100, 100, 100), nnz=10_000, seed=1001, kind=0),
        # permute = 1 (R#22): labels relabelled by pi_k, then re-sorted; odd and 2^k dims
        dict(dims=(12092, 9184, 28818), nnz=100_000, seed=1002, permute=1),
        dict(dims=(1 << 12, 1 << 12, 1 << 12), nnz=50_000, seed=9, permute=1),
    ]
    for c in cases:
        kind = c.get("kind", 1)
        x = pasta.pasta_gen_powerlaw(c["dims"], c["nnz"], c["seed"], kind=kind,
                                     initiator=c.get("initiator"), permute=c.get("permute", 0))
        gi, gv = pasta.pasta_coo_export(x)
        oi, ov = oracle.gen_powerlaw(c["dims"], c["nnz"], c["seed"], initiator=c.get("initiator"),
                                     q=0.5 if kind == 0 else 0.75, permute=bool(c.get("permute", 0)))
        np.testing.assert_array_equal(gi, oi)
        np.testing.assert_array_equal(gv.view(np.uint32), ov.view(np.uint32))


def test_mode_sort_bit_exact_with_oracle(env):
    pasta, oracle, torch = env
    dims = (3000, 200, 4000, 50)
    inds, vals = si.powerlaw_coo(dims, 100_000, seed=4)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    for n in range(4):
        gi, gv = pasta.pasta_coo_export_mode(x, n)
        oi, ov = oracle.mode_sort(inds, vals, n)
        np.testing.assert_array_equal(gi, oi)
        np.testing.assert_array_equal(gv.view(np.uint32), ov.view(np.uint32))


@pytest.mark.parametrize("dims,nnz,bb", [((300, 200, 500), 50_013, 7), ((60, 70, 80, 90), 40_007, 4),
                                         ((4096, 4096, 4096), 200_000, 7), ((1000, 900), 30_001, 1),
                                         ((1 << 20, 3, 1 << 12), 30_000, 8)])
def test_hicoo_conversion_bit_exact(env, dims, nnz, bb):
    pasta, oracle, torch = env
    inds, vals = si.powerlaw_coo(dims, nnz, seed=nnz)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_hicoo_export(pasta.pasta_coo_to_hicoo(x, bb))
    o = oracle.coo_to_hicoo(inds, vals, bb)
    assert h["nblocks"] == o["nblocks"]
    np.testing.assert_array_equal(h["bptr"], o["bptr"])
    np.testing.assert_array_equal(h["binds"], o["binds"])
    np.testing.assert_array_equal(h["einds"], o["einds"])
    np.testing.assert_array_equal(h["vals"].view(np.uint32), o["vals"].view(np.uint32))


def test_shards_cover_the_output(env):
    pasta, oracle, torch = env
    dims = (2000, 300, 400)
    inds, vals = si.hot_row_coo(dims, 20_000, 60_000, seed=9, mode=1, hot_row=17)
    U = si.factors(dims, 16, seed=4)
    Ud = _dev(torch, U)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    for n in range(3):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        counts = pasta.pasta_coo_row_counts(x, n)
        np.testing.assert_array_equal(counts, np.bincount(inds[n], minlength=dims[n]))
        for P in (1, 3, 8):
            bounds = pasta.pasta_coo_partition(x, n, P)
            np.testing.assert_array_equal(bounds, pasta.pasta_row_partition(counts, P))
            out = torch.full((dims[n], 16), float("nan"), device="cuda")
            total = 0
            for p in range(P):
                s = pasta.pasta_coo_shard(x, n, int(bounds[p]), int(bounds[p + 1]))
                total += s.nnz
                pasta.pasta_mttkrp_coo(s, n, Ud, out=out)  # writes only its rows
            assert total == vals.shape[0]
            _check(out, ref, ab, f"shards mode {n} P={P}")
        # the full sorted copy freed after sharding is rebuilt on the next use
        pasta.pasta_coo_release_mode(x, n)
        _check(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, f"after release mode {n}")


@pytest.mark.parametrize("cmask", [0b111, 0b101])
def test_hicoo_shards_bit_exact_and_cover_the_output(env, cmask):
    """pasta_hicoo_shard: every shard equals the oracle's conversion of the
    COO sub-tensor of its rows, bit for bit; the shards' MTTKRPs write disjoint row ranges
    that together give the full result.  cmask 0b101: gHiCOO with mode 1 uncompressed."""
    pasta, oracle, torch = env
    dims = (2000, 300, 400)
    inds, vals = si.hot_row_coo(dims, 20_000, 60_000, seed=9, mode=1, hot_row=17)
    U = si.factors(dims, 16, seed=4)
    Ud = _dev(torch, U)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    h = pasta.pasta_coo_to_hicoo(x, 7) if cmask == 0b111 else pasta.pasta_coo_to_ghicoo(x, 7, cmask)
    for n in range(3):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        bounds = pasta.pasta_coo_partition(x, n, 3)
        out = torch.full((dims[n], 16), float("nan"), device="cuda")
        total = 0
        for p in range(3):
            lo, hi = int(bounds[p]), int(bounds[p + 1])
            sh = pasta.pasta_hicoo_shard(h, n, lo, hi)
            total += sh.nnz
            mine = (inds[n] >= lo) & (inds[n] < hi)
            si_, sv_ = np.ascontiguousarray(inds[:, mine]), vals[mine]
            if cmask == 0b111:
                got, want = pasta.pasta_hicoo_export(sh), oracle.coo_to_hicoo(si_, sv_, 7)
                keys = ("bptr", "binds", "einds")
                for k in keys:
                    assert np.array_equal(got[k], want[k]), (n, p, k)
            else:
                got, want = pasta.pasta_ghicoo_export(sh), oracle.coo_to_ghicoo(si_, sv_, 7, cmask)
                assert np.array_equal(got["bptr"], want["bptr"]), (n, p)
                for k in range(3):
                    for key in ("binds", "einds", "uinds"):
                        if want[key][k] is not None:
                            assert np.array_equal(got[key][k], want[key][k]), (n, p, key, k)
            assert got["nblocks"] == want["nblocks"]
            assert np.array_equal(got["vals"].view(np.uint32), want["vals"].view(np.uint32))
            pasta.pasta_mttkrp_hicoo(sh, n, Ud, out=out)  # writes only its rows
        assert total == vals.shape[0]
        _check(out, ref, ab, f"hicoo shards mode {n}")


def test_allmodes_host_e2e_matches_device(env):
    pasta, oracle, torch = env
    dims = (500, 400, 300)
    inds, vals = si.powerlaw_coo(dims, 60_000, seed=11)
    U = si.factors(dims, 16, seed=12)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    hf = [torch.from_numpy(u).pin_memory() for u in U]
    ho = [torch.empty((d, 16), dtype=torch.float32).pin_memory() for d in dims]
    pasta.pasta_mttkrp_coo_allmodes_host(x, hf, ho)
    for n in range(3):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        _check(ho[n].numpy().astype(np.float64), ref, ab, f"e2e mode {n}")


def test_allmodes_host_batch_pipelined_steps(env):
    """pasta_mttkrp_coo_allmodes_host_batch: independent steps with different factors share two
    device staging slots (step i+1 uploads while step i downloads); every step's result must
    match the oracle for that step's factors (a slot reused too early would mix steps)."""
    pasta, oracle, torch = env
    dims = (700, 500, 900)
    inds, vals = si.powerlaw_coo(dims, 80_000, seed=21)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    steps, Us = [], []
    for i in range(5):
        U = si.factors(dims, 16, seed=100 + i)
        Us.append(U)
        hf = [torch.from_numpy(u).pin_memory() for u in U]
        ho = [torch.full((d, 16), float("nan"), dtype=torch.float32).pin_memory() for d in dims]
        steps.append((hf, ho))
    pasta.pasta_mttkrp_coo_allmodes_host_batch(x, steps)
    for i, (hf, ho) in enumerate(steps):
        for n in range(3):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, Us[i])
            _check(ho[n].numpy().astype(np.float64), ref, ab, f"batch step {i} mode {n}")
    pasta.pasta_mttkrp_coo_allmodes_host_batch(x, [])  # no-op


def test_tns_roundtrip(env, tmp_path):
    pasta, oracle, torch = env
    dims = (50, 60, 70)
    inds, vals = si.uniform_coo(dims, 2000, seed=2)
    p = tmp_path / "t.tns"
    with open(p, "w") as f:
        f.write("# FROSTT-style, 1-based\n")
        for x in range(vals.shape[0]):
            f.write(" ".join(str(int(inds[k, x]) + 1) for k in range(3)) + f" {float(vals[x]):.9g}\n")
    t = pasta.pasta_load_coo(str(p))
    assert t.order == 3 and t.nnz == 2000
    assert t.dims == tuple(int(inds[k].max()) + 1 for k in range(3))
    gi, gv = pasta.pasta_coo_export(t)
    np.testing.assert_array_equal(gi, inds)
    np.testing.assert_array_equal(gv, vals)
    q = tmp_path / "u.tns"
    pasta.pasta_save_coo(t, str(q))
    t2 = pasta.pasta_load_coo(str(q))
    gi2, gv2 = pasta.pasta_coo_export(t2)
    np.testing.assert_array_equal(gi2, inds)
    np.testing.assert_array_equal(gv2, vals)
    # binary cache (.pbin): bit-exact round trip, stored dims kept (larger than the max index)
    big = pasta.pasta_coo_from_arrays((70, 80, 90), inds, vals)
    b = tmp_path / "t.pbin"
    pasta.pasta_save_coo(big, str(b))
    assert b.read_bytes()[:8] == b"PASTAB01"
    assert b.stat().st_size == 8 + 16 + 12 + 4 * 4 * 2000
    t3 = pasta.pasta_load_coo(str(b))
    assert t3.dims == (70, 80, 90) and t3.nnz == 2000
    gi3, gv3 = pasta.pasta_coo_export(t3)
    np.testing.assert_array_equal(gi3, inds)
    np.testing.assert_array_equal(gv3.view(np.uint32), vals.view(np.uint32))


def test_misaligned_factor_takes_scalar_path(env):
    pasta, oracle, torch = env
    dims = (300, 200, 100)
    inds, vals = si.uniform_coo(dims, 20_000, seed=8)
    U = si.factors(dims, 16, seed=8)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    Ud = []
    for u in U:  # a view starting 4 bytes into a buffer: not 16-byte aligned
        buf = torch.empty(u.size + 1, dtype=torch.float32, device="cuda")
        v = buf[1:].view(u.shape)
        v.copy_(torch.from_numpy(u))
        Ud.append(v)
    for n in range(3):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        _check(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, f"misaligned mode {n}")


def test_profile_and_launch_counters(env):
    pasta, oracle, torch = env
    dims = (300, 200, 100)
    inds, vals = si.uniform_coo(dims, 20_000, seed=8)
    Ud = _dev(torch, si.factors(dims, 16, seed=8))
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    pasta.pasta_mttkrp_coo(x, 0, Ud)
    pasta.pasta_profile_read(0, reset=True)
    pasta.pasta_profile_enable(True)
    n0 = pasta.pasta_launch_count()
    pasta.pasta_mttkrp_coo(x, 0, Ud)
    per_call = pasta.pasta_launch_count() - n0  # zero-fill (+ hot-row fills) + MTTKRP
    for _ in range(2):
        pasta.pasta_mttkrp_coo(x, 0, Ud)
    ms, n = pasta.pasta_profile_read(0, reset=True)
    pasta.pasta_profile_enable(False)
    assert n == 3 and ms > 0
    assert 2 <= per_call <= 2 + len(dims) - 1
    assert pasta.pasta_launch_count() - n0 == 3 * per_call


def test_errors_on_device(env):
    pasta, oracle, torch = env
    dims = (10, 10, 10)
    x = pasta.pasta_coo_from_arrays(dims, np.zeros((3, 1), np.uint32), np.ones(1, np.float32))
    Ud = _dev(torch, si.factors(dims, 4, seed=0))
    with pytest.raises(pasta.PastaError):
        pasta.pasta_mttkrp_coo(x, 3, Ud)
    with pytest.raises(pasta.PastaError):
        pasta.pasta_coo_to_hicoo(x, 9)
    with pytest.raises(pasta.PastaError):
        pasta.pasta_coo_shard(x, 0, 5, 3)


@pytest.mark.parametrize("heavy", ["128", "16"])
def test_hicoo_block_layout_with_tma_staged_heavy_blocks(env, heavy, monkeypatch):
    """The block-major HiCOO copy (PASTA_HICOO_LAYOUT=block): heavy blocks are processed one
    per CTA from factor tiles staged in shared memory by TMA bulk copies, light blocks by the
    warp-run kernel.  Same tolerance as every other path."""
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_HICOO_LAYOUT", "block")
    monkeypatch.setenv("PASTA_HICOO_HEAVY", heavy)
    for dims, nnz, R, bb in [((300, 200, 500), 50_013, 16, 7), ((60, 70, 80, 90), 40_007, 32, 4),
                             ((5000, 3000, 2000), 200_000, 16, 7)]:
        inds, vals = si.powerlaw_coo(dims, nnz, seed=nnz)
        U = si.factors(dims, R, seed=3)
        Ud = _dev(torch, U)
        x = pasta.pasta_coo_from_arrays(dims, inds, vals)
        h = pasta.pasta_coo_to_hicoo(x, bb)
        for n in range(len(dims)):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
            _check(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab, f"block layout {dims} mode {n}")


def test_row_partitioned_runner_two_ranks_on_one_gpu(env):
    """parallel.RowPartitionedMTTKRP for world = 2, both ranks simulated on this GPU without a
    process group (gather=False): the union of each rank's owned rows equals the oracle."""
    pasta, oracle, torch = env
    from paper_conf_iiswc_lilwlob20_b200.parallel import RowPartitionedMTTKRP
    dims = (3000, 800, 1200)
    inds, vals = si.hot_row_coo(dims, 50_000, 150_000, seed=21, mode=2, hot_row=5)
    U = si.factors(dims, 16, seed=6)
    Ud = _dev(torch, U)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    parts = [RowPartitionedMTTKRP(x, r, 2, 16, torch.device("cuda")) for r in range(2)]
    assert sum(sum(p.shard_nnz()) for p in parts) == 3 * vals.shape[0]
    outs = [p.step(Ud, gather=False) for p in parts]
    for n in range(3):
        ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
        full = torch.empty((dims[n], 16), device="cuda")
        for r in range(2):
            lo, hi = int(parts[r].bounds[n][r]), int(parts[r].bounds[n][r + 1])
            full[lo:hi] = outs[r][n][lo:hi]
        _check(full, ref, ab, f"rank-partitioned mode {n}")


def test_torch_caching_allocator_hook(env):
    """pasta_set_allocator: every libpasta device allocation goes through torch's caching
    allocator (use_torch_allocator); results unchanged, memory visible to torch."""
    pasta, oracle, torch = env
    dims = (500, 400, 300)
    inds, vals = si.powerlaw_coo(dims, 60_000, seed=2)
    U = si.factors(dims, 16, seed=2)
    Ud = _dev(torch, U)
    torch.cuda.synchronize()
    before = torch.cuda.memory_allocated()
    pasta.use_torch_allocator()
    try:
        x = pasta.pasta_coo_from_arrays(dims, inds, vals)
        h = pasta.pasta_coo_to_hicoo(x, 7)
        g = pasta.pasta_gen_powerlaw((1000, 1000, 1000), 50_000, seed=3)
        for n in range(3):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
            _check(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, f"hooked coo mode {n}")
            _check(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab, f"hooked hicoo mode {n}")
        assert torch.cuda.memory_allocated() > before  # the handles' arrays live in torch's pool
        del x, h, g
        import gc
        gc.collect()
    finally:
        pasta.pasta_set_allocator(None)


@pytest.mark.parametrize("hot_mb,persist", [("0.05", "0"), ("1", "0"), ("1", "1")])
def test_coo_hot_row_cache_forced(env, hot_mb, persist, monkeypatch):
    """The packed hot-row cache (coo_mark_hot) is enabled automatically only when the gathered
    factors exceed L2; force it on small tensors (tiny budgets so that hot and cold rows mix),
    with and without the persisting-L2 access-policy window (a separate launch path)."""
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_HOT_FORCE", "1")
    monkeypatch.setenv("PASTA_HOT_MB", hot_mb)
    monkeypatch.setenv("PASTA_HOT_PERSIST", persist)
    for dims, nnz, R in [((3000, 2000, 4000), 120_000, 16), ((300, 400, 500, 60), 80_000, 32),
                         ((5000, 3000, 2000), 0, 16)]:
        if nnz:
            inds, vals = si.powerlaw_coo(dims, nnz, seed=nnz + R)
        else:
            inds, vals = si.hot_row_coo(dims, 300_000, 50_000, seed=4, mode=1, hot_row=0)
        U = si.factors(dims, R, seed=R)
        Ud = _dev(torch, U)
        x = pasta.pasta_coo_from_arrays(dims, inds, vals)
        for n in range(len(dims)):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
            _check(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, f"hot cache {dims} R={R} mode {n}")
        # factors change between calls (CP-ALS): the cache is refilled every launch
        Ud2 = [u * 0.5 for u in Ud]
        U2 = [u.cpu().numpy() for u in Ud2]
        ref, ab = oracle.mttkrp(dims, inds, vals, 0, U2)
        _check(pasta.pasta_mttkrp_coo(x, 0, Ud2), ref, ab, "hot cache refill")


@pytest.mark.parametrize("l2_tier,hs_cfg", [(False, "0"), (True, "0"), (False, "1"), (True, "1"), (True, "2")])
def test_coo_shared_memory_hot_tier(env, l2_tier, hs_cfg, monkeypatch):
    """The shared-memory tier of the hot-row cache (persistent coo_staged_kernel<..., HS>):
    forced on, alone or together with a tiny L2 tier so that smem-, L2-tier- and cold rows
    mix in one warp; 3M nonzeros give every warp of the persistent grid several chunks.
    Every kernel shape (16 warps x 32-deep stages, 24 warps x 16-deep, 8 nonzeros per group
    step) for every order."""
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_HOT_SMEM", "1")
    monkeypatch.setenv("PASTA_HS_CFG", hs_cfg)
    if l2_tier:
        monkeypatch.setenv("PASTA_HOT_FORCE", "1")
        monkeypatch.setenv("PASTA_HOT_MB", "0.25")
    for dims, nnz, R in [((3000, 2000, 4000), 3_000_017, 16), ((300, 400, 500, 60), 80_000, 16),
                         ((3000, 2000, 4000), 120_000, 32), ((300, 400, 500, 60), 80_000, 32),
                         ((3000, 2000, 4000), 200_000, 8), ((3000, 2000, 4000), 200_000, 64),
                         ((5000, 3000, 2000), 0, 16)]:
        if nnz:
            inds, vals = si.powerlaw_coo(dims, nnz, seed=nnz + R)
        else:
            inds, vals = si.hot_row_coo(dims, 300_000, 50_000, seed=4, mode=1, hot_row=0)
        U = si.factors(dims, R, seed=R)
        Ud = _dev(torch, U)
        x = pasta.pasta_coo_from_arrays(dims, inds, vals)
        for n in range(len(dims)):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
            _check(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, f"smem tier {dims} R={R} mode {n}")
        Ud2 = [u * 0.5 for u in Ud]  # the tier is re-read from the factors at every launch
        U2 = [u.cpu().numpy() for u in Ud2]
        ref, ab = oracle.mttkrp(dims, inds, vals, 1, U2)
        _check(pasta.pasta_mttkrp_coo(x, 1, Ud2), ref, ab, "smem tier refill")


@pytest.mark.parametrize("staged", ["1", "0", "raw"])
def test_hicoo_row_slices_staged_decode(env, staged, monkeypatch):
    """HiCOO / gHiCOO row-slice MTTKRP with the slices decoded warp-wide into the staged kernel
    (default) and with the per-group slice walk (PASTA_HICOO_STAGED=0): hypersparse blocks
    (~1 entry per slice, a window spans 32 slices), dense blocks (long slices), a 300K-entry
    hot row (slices longer than any window), R = 16 / 32, orders 2-4, gHiCOO masks with
    uncompressed (32-bit) modes, and enough nonzeros for several chunks per persistent warp."""
    pasta, oracle, torch = env
    monkeypatch.setenv("PASTA_HICOO_STAGED", "0" if staged == "0" else "1")
    monkeypatch.setenv("PASTA_HICOO_RAW", "1" if staged == "raw" else "0")  # WA 11 raw-staged decode
    cases = [((1 << 20, 1 << 20, 1 << 20), 400_000, 16, "powerlaw", 7, None),
             ((300, 200, 500), 2_500_000, 16, "uniform", 7, None),
             ((600, 500, 400), 200_000, 32, "uniform", 5, None),
             ((2000, 1500), 150_000, 16, "powerlaw", 6, None),
             ((60, 70, 80, 90), 300_000, 16, "powerlaw", 4, None),
             ((3000, 2000, 4000), 300_000, 16, "powerlaw", 7, 0b101),
             ((3000, 2000, 4000), 300_000, 32, "powerlaw", 7, 0b010),
             ((3000, 2000, 4000), 200_000, 8, "powerlaw", 7, None),
             ((3000, 2000, 4000), 200_000, 64, "powerlaw", 7, None),
             ((60, 70, 80, 90), 100_000, 64, "powerlaw", 4, 0b1011),
             ((5000, 3000, 2000), 0, 16, "hot", 7, None)]
    for dims, nnz, R, gen, bb, mask in cases:
        if gen == "hot":
            inds, vals = si.hot_row_coo(dims, 300_000, 50_000, seed=8, mode=0, hot_row=7)
        else:
            mk = si.powerlaw_coo if gen == "powerlaw" else si.uniform_coo
            inds, vals = mk(dims, nnz, seed=nnz + R + bb)
        U = si.factors(dims, R, seed=R + 1)
        Ud = _dev(torch, U)
        x = pasta.pasta_coo_from_arrays(dims, inds, vals)
        h = pasta.pasta_coo_to_ghicoo(x, bb, mask) if mask else pasta.pasta_coo_to_hicoo(x, bb)
        for n in range(len(dims)):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
            _check(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab,
                   f"hicoo staged={staged} {dims} R={R} mask={mask} mode {n}")


@pytest.mark.parametrize("split", ["1", "0"])
def test_coo_die_split(env, split, monkeypatch):
    """Die-split COO MTTKRP (R#35): with the L2 tier forced on, order-3 nonzeros are reordered
    into four row-sorted segments by the die halves of their two gathered rows and the
    persistent kernel's CTAs claim chunks of their die's range; every flush is an atomic.
    Checked against the oracle for both settings on the same handle (the ranking is redone
    when the split changes), with a 1M-nonzero hot row crossing all four segments."""
    pasta, oracle, torch = env
    die, nd = pasta.pasta_die_map()
    assert die is not None and min(nd) >= 148 // 3, nd  # a plausible two-die B200 split
    assert np.count_nonzero(die == 0) == nd[0] and np.count_nonzero(die == 1) == nd[1]
    monkeypatch.setenv("PASTA_HOT_FORCE", "1")
    monkeypatch.setenv("PASTA_HOT_MB", "0.5")
    monkeypatch.setenv("PASTA_DIE_SPLIT", split)
    for dims, nnz, R in [((3000, 2000, 4000), 2_000_003, 16), ((4000, 900, 2500), 0, 32)]:
        if nnz:
            inds, vals = si.powerlaw_coo(dims, nnz, seed=nnz + R)
        else:
            inds, vals = si.hot_row_coo(dims, 1_000_000, 200_000, seed=8, mode=0, hot_row=17)
        U = si.factors(dims, R, seed=R)
        Ud = _dev(torch, U)
        x = pasta.pasta_coo_from_arrays(dims, inds, vals)
        for n in range(3):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
            _check(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, f"die split {split} {dims} R={R} mode {n}")
        monkeypatch.setenv("PASTA_DIE_SPLIT", "1" if split == "0" else "0")  # flip on the same handle
        ref, ab = oracle.mttkrp(dims, inds, vals, 2, U)
        _check(pasta.pasta_mttkrp_coo(x, 2, Ud), ref, ab, f"die split flipped {dims} R={R}")
        monkeypatch.setenv("PASTA_DIE_SPLIT", split)
