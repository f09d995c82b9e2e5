#!/usr/bin/env python
"""TS / TEW kernel variant sweep (PASTA_EW_VARIANT) on 100M-element value arrays: GB/s per
Table I's bytes (TS 8 B, TEW 12 B per element)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_iiswc_lilwlob20_b200 as pasta  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 100_000_000
a = torch.rand(n, device="cuda")
b = torch.rand(n, device="cuda")
o = torch.empty_like(a)
for name, fn, nb in (("ts_mul", lambda: pasta.pasta_ts(a, "mul", 0.5, out=o), 8 * n),
                     ("tew_add", lambda: pasta.pasta_tew(a, b, "add", out=o), 12 * n),
                     ("torch_copy", lambda: o.copy_(a), 8 * n)):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        fn()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 20
    print(json.dumps({"variant": os.environ.get("PASTA_EW_VARIANT", "0"), "kernel": name,
                      "ms": round(ms, 4), "GB/s": round(nb / ms / 1e6, 1)}), flush=True)
