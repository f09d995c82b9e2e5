import sys, os; sys.path.insert(0, '.')
import numpy as np, torch
import paper_conf_iiswc_lilwlob20_b200 as pasta, synth_inputs as si
cfg = si.CONFIGS["h"]
x = pasta.pasta_gen_powerlaw(cfg["dims"], cfg["nnz"], cfg["seed"])
U = [torch.rand((d, 16), device="cuda") for d in cfg["dims"]]
pasta.pasta_mttkrp_coo(x, 0, U); torch.cuda.synchronize()
c1 = pasta.pasta_coo_row_counts(x, 1).astype(np.int64)
s = np.sort(c1)[::-1]
cum = np.cumsum(s) / s.sum()
for k in [100_000, 300_000, 524_288, 1_000_000, 2_000_000]:
    print("top", k, "rows of factor 1 cover", round(cum[k-1], 3), "of accesses; count at k:", s[k-1])
print("nonzero rows", (c1 > 0).sum(), "max", s[0])
