import os, sys
import numpy as np, torch
sys.path.insert(0, os.getcwd())
import synth_inputs as si
import paper_conf_iiswc_lilwlob20_b200 as pasta
import oracle
cfg, R, tier, dims = sys.argv[1], int(sys.argv[2]), sys.argv[3], tuple(int(v) for v in sys.argv[4].split("x"))
os.environ.update(PASTA_HICOO_HOT=tier, PASTA_HOT_FORCE="1", PASTA_HOT_MB="0.2", PASTA_HS_CFG=cfg)
inds, vals = si.powerlaw_coo(dims, 120_000, seed=5)
x = pasta.pasta_coo_from_arrays(dims, inds, vals)
h = pasta.pasta_coo_to_hicoo(x, 7)
U = si.factors(dims, R, seed=R + 11)
Ud = [torch.from_numpy(u).cuda() for u in U]
for n in range(len(dims)):
    ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
    got = pasta.pasta_mttkrp_hicoo(h, n, Ud).cpu().numpy()
    ex = np.abs(got - ref) - (1e-4 * ab + 1e-6)
    print(cfg, R, tier, dims, n, "max excess", ex.max(), flush=True)
