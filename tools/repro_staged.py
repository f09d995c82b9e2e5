import sys; sys.path.insert(0, '.')
import numpy as np, torch
import paper_conf_iiswc_lilwlob20_b200 as pasta, synth_inputs as si
dims=(300,200,500); inds, vals = si.uniform_coo(dims, 50013, seed=1)
R=int(sys.argv[1]) if len(sys.argv)>1 else 32
U=[torch.from_numpy(u).cuda() for u in si.factors(dims, R, seed=1)]
x=pasta.pasta_coo_from_arrays(dims, inds, vals)
o=pasta.pasta_mttkrp_coo(x, 0, U); torch.cuda.synchronize(); print("ok", o.sum().item())
