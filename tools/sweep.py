#!/usr/bin/env python
"""Tuning sweep of MTTKRP kernel variants (PASTA_MTTKRP_VARIANT / PASTA_MTTKRP_RUN) on one
bench workload.  Prints one JSON line per (format, variant, run): mean kernel ms per mode."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_iiswc_lilwlob20_b200 as pasta  # noqa: E402
import synth_inputs as si  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="h")
    ap.add_argument("--variants", default="0,1,2,3,4,5,6,7")
    ap.add_argument("--runs", default="128")
    ap.add_argument("--formats", default="coo")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--caches", default="", help="PASTA_MTTKRP_CACHE values (default: leave the env)")
    ap.add_argument("--cmask", type=int, default=0, help="gHiCOO mask (0 = auto)")
    ap.add_argument("--R", type=int, default=0, help="override the config's rank")
    args = ap.parse_args()
    cfg = si.CONFIGS[args.config]
    dims, R, M = cfg["dims"], cfg["R"], cfg["nnz"]
    R = args.R or R
    x = pasta.pasta_gen_powerlaw(dims, M, cfg["seed"], kind=0 if cfg["kind"] == "uniform" else 1)
    fmts = args.formats.split(",")
    h = pasta.pasta_coo_to_hicoo(x, 7) if "hicoo" in fmts else None
    gh = pasta.pasta_coo_to_ghicoo(x, 7, args.cmask) if "ghicoo" in fmts else None
    if gh is not None:
        print(json.dumps({"ghicoo_cmask": gh.cmask, "ghicoo_nblocks": gh.nblocks}), flush=True)
    g = torch.Generator(device="cuda")
    g.manual_seed(1)
    U = [torch.rand((d, R), generator=g, device="cuda") for d in dims]
    outs = [torch.empty((d, R), device="cuda") for d in dims]
    if h is not None:
        print(json.dumps({"hicoo_nblocks": h.nblocks, "nnz": h.nnz}), flush=True)
    for fmt in fmts:
        fn, t = {"coo": (pasta.pasta_mttkrp_coo, x), "hicoo": (pasta.pasta_mttkrp_hicoo, h),
                 "ghicoo": (pasta.pasta_mttkrp_hicoo, gh)}[fmt]
        which = 0 if fmt == "coo" else 1
        for n in range(len(dims)):
            fn(t, n, U, out=outs[n])  # prepare
        caches = args.caches.split(",") if args.caches else [os.environ.get("PASTA_MTTKRP_CACHE", "0")]
        combos = [(r, v, c) for r in args.runs.split(",") for v in args.variants.split(",")
                  for c in caches]
        for run, var, cache in [(int(r), int(v), int(c)) for r, v, c in combos]:
            if True:
                os.environ["PASTA_MTTKRP_CACHE"] = str(cache)
                os.environ["PASTA_MTTKRP_VARIANT"] = str(var)
                if run:
                    os.environ["PASTA_MTTKRP_RUN"] = str(run)
                else:  # 0: the library's default for the regime
                    os.environ.pop("PASTA_MTTKRP_RUN", None)
                per_mode = []
                for n in range(len(dims)):
                    for _ in range(2):
                        fn(t, n, U, out=outs[n])
                    torch.cuda.synchronize()
                    pasta.pasta_profile_read(which, reset=True)
                    pasta.pasta_profile_enable(True)
                    for _ in range(args.reps):
                        fn(t, n, U, out=outs[n])
                    torch.cuda.synchronize()
                    pasta.pasta_profile_enable(False)
                    ms, k = pasta.pasta_profile_read(which, reset=True)
                    per_mode.append(round(ms / k, 4))
                print(json.dumps({"config": args.config, "fmt": fmt, "variant": var, "run": run, "cache": cache,
                                  "ms_per_mode": per_mode,
                                  "mean_ms": round(sum(per_mode) / len(per_mode), 4)}), flush=True)


if __name__ == "__main__":
    main()
