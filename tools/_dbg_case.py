import os, sys
import numpy as np, torch
import synth_inputs as si
import paper_conf_iiswc_lilwlob20_b200 as pasta
import oracle
dims = tuple(int(v) for v in sys.argv[1].split("x")); R = int(sys.argv[2])
inds, vals = si.powerlaw_coo(dims, 120_000, seed=5)
x = pasta.pasta_coo_from_arrays(dims, inds, vals)
h = pasta.pasta_coo_to_hicoo(x, 7)
U = si.factors(dims, R, seed=R + 11)
Ud = [torch.from_numpy(u).cuda() for u in U]
worst = -1.0
for n in range(len(dims)):
    ref, ab = oracle.mttkrp(dims, inds, vals, n, U)
    got = pasta.pasta_mttkrp_hicoo(h, n, Ud).cpu().numpy()
    worst = max(worst, float((np.abs(got - ref) - (1e-4 * ab + 1e-6)).max()))
print("OK" if worst <= 0 else f"WRONG {worst:.3e}")
