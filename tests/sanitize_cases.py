#!/usr/bin/env python
"""Tiny cases over every kernel family, checked against the oracle, for compute-sanitizer
(SURVEY section 4 item 8):

  compute-sanitizer --tool memcheck|racecheck|synccheck --error-exitcode 9 \
      python tests/sanitize_cases.py

COO MTTKRP (N = 3, 4; R = 8, 16, 32; default and forced hot-row cache, die split), HiCOO
(staged decode, raw-staged decode, hot-block tiers, shards) and gHiCOO MTTKRP, mode sort,
TTV / TTM, CP-ALS (incl. the fit kernel), TS / TEW, both generators (with relabelling)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_iiswc_lilwlob20_b200 as pasta  # noqa: E402
import synth_inputs as si  # noqa: E402


def close(got, ref, ab, what):
    g = got.detach().cpu().numpy().astype(np.float64)
    assert np.all(np.abs(g - ref) <= 1e-4 * ab + 1e-6), what


def main():
    torch.cuda.set_device(0)
    cases = [((60, 70, 80), 3000, 16), ((300, 40, 500), 5000, 32), ((50, 60, 70), 2000, 8),
             ((20, 30, 40, 50), 4000, 16)]
    for dims, nnz, R in cases:
        inds, vals = si.powerlaw_coo(dims, nnz, seed=7)
        U = si.factors(dims, R, seed=8)
        Ud = [torch.from_numpy(u).cuda() for u in U]
        x = pasta.pasta_coo_from_arrays(dims, inds, vals)
        h = pasta.pasta_coo_to_hicoo(x, 3)
        g = pasta.pasta_coo_to_ghicoo(x, 3, 1)
        for n in range(len(dims)):
            ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
            for force in ("0", "1"):
                os.environ["PASTA_HOT_FORCE"] = force
                close(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, (dims, R, n, "coo", force))
            if len(dims) == 3:  # die-split COO (R#35), forced
                os.environ["PASTA_HOT_FORCE"] = "1"
                os.environ["PASTA_DIE_SPLIT"] = "1"
                close(pasta.pasta_mttkrp_coo(x, n, Ud), ref, ab, (dims, R, n, "coo split"))
                os.environ["PASTA_DIE_SPLIT"] = "0"
            os.environ["PASTA_HOT_FORCE"] = "0"
            close(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab, (dims, R, n, "hicoo"))
            for env in ("PASTA_HICOO_RAW", "PASTA_HICOO_HOT"):  # WA 11 raw decode, WA 10 hot blocks
                os.environ[env] = "1"
                close(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab, (dims, R, n, "hicoo", env))
                os.environ[env] = "0"
            # R#36 tier blocks: smem tier only (WA 17), then smem + L2 tiers forced (WA 10)
            os.environ["PASTA_HICOO_HOT"] = "2"
            for force in ("0", "1"):
                os.environ["PASTA_HOT_FORCE"] = force
                close(pasta.pasta_mttkrp_hicoo(h, n, Ud), ref, ab, (dims, R, n, "hicoo tier blocks", force))
            os.environ["PASTA_HOT_FORCE"] = "0"
            os.environ["PASTA_HICOO_HOT"] = "0"
            bounds = pasta.pasta_coo_partition(x, n, 2)
            out = torch.zeros((dims[n], R), device="cuda")
            for p in range(2):
                pasta.pasta_mttkrp_hicoo(pasta.pasta_hicoo_shard(h, n, int(bounds[p]), int(bounds[p + 1])), n, Ud,
                                         out=out)
            close(out, ref, ab, (dims, R, n, "hicoo shards"))
            close(pasta.pasta_mttkrp_hicoo(g, n, Ud), ref, ab, (dims, R, n, "ghicoo"))
            si_, sv_ = pasta.pasta_coo_export_mode(x, n)
            oi, ov = oracle.mode_sort(inds, vals, n)
            assert np.array_equal(si_, oi) and np.array_equal(sv_, ov), (dims, n, "sort")
            f, y, ya = oracle.ttm(dims, inds, vals, n, U[n])
            close(pasta.pasta_ttm_coo(x, n, Ud[n]), y, ya, (dims, n, "ttm"))
            v = U[n][:, 0].copy()
            f, y, ya = oracle.ttv(dims, inds, vals, n, v)
            close(pasta.pasta_ttv_coo(x, n, torch.from_numpy(v).cuda()), y, ya, (dims, n, "ttv"))
        print("ok", dims, R, flush=True)

    # CP-ALS: 3 sweeps from the same init as the oracle
    from oracle.cpals import cp_als
    dims, R = (40, 50, 60), 8
    inds, vals = si.powerlaw_coo(dims, 3000, seed=11)
    U0 = si.factors(dims, R, seed=12)
    x = pasta.pasta_coo_from_arrays(dims, inds, vals)
    Ud = [torch.from_numpy(u.copy()).cuda() for u in U0]
    Uo, lam_o, fits_o = cp_als(dims, inds, vals, U0, iters=3)
    lam, fits, it = pasta.pasta_cpals_coo(x, Ud, max_iters=3, tol=0.0)
    assert it == 3 and np.allclose(fits, fits_o, atol=2e-4), (fits, fits_o)
    assert np.allclose(lam, lam_o, rtol=2e-3)
    print("ok cpals", flush=True)

    # TS / TEW on a ragged length
    a = torch.rand(100_003, device="cuda") + 0.5
    b = torch.rand(100_003, device="cuda") + 0.5
    for op in ("add", "sub", "mul", "div"):
        got = pasta.pasta_ts(a, op, 1.5).cpu().numpy()
        assert np.array_equal(got, oracle.ts(a.cpu().numpy(), op, 1.5)), op
        got = pasta.pasta_tew(a, b, op).cpu().numpy()
        assert np.array_equal(got, oracle.tew_same(a.cpu().numpy(), b.cpu().numpy(), op)), op
    print("ok ts/tew", flush=True)

    # generators (kind 1 Kronecker, kind 2 slice power law), bit-exact vs the oracle
    for kind, fn in ((1, oracle.gen_powerlaw), (2, oracle.gen_slice_powerlaw)):
        dims = (1000, 700, 33)
        x = pasta.pasta_gen_powerlaw(dims, 5000, 3, kind=kind)
        gi, gv = pasta.pasta_coo_export(x)
        oi, ov = fn(dims, 5000, 3)
        assert np.array_equal(gi, oi) and np.array_equal(gv, ov), kind
    x = pasta.pasta_gen_powerlaw((1000, 700, 33), 5000, 3, permute=1)  # relabelled (R#22)
    gi, gv = pasta.pasta_coo_export(x)
    oi, ov = oracle.gen_powerlaw((1000, 700, 33), 5000, 3, permute=True)
    assert np.array_equal(gi, oi) and np.array_equal(gv, ov), "permute"
    print("ok generators", flush=True)
    torch.cuda.synchronize()
    print("sanitize cases done", flush=True)


if __name__ == "__main__":
    main()
