"""Run CP-ALS sweeps on a bench workload (for profiling the CP-ALS kernels)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_iiswc_lilwlob20_b200 as pasta
import synth_inputs as si
cfg = si.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "h"]
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 2
x = pasta.pasta_gen_powerlaw(cfg["dims"], cfg["nnz"], cfg["seed"])
g = torch.Generator(device="cuda"); g.manual_seed(1)
U = [torch.rand((d, cfg["R"]), generator=g, device="cuda") for d in cfg["dims"]]
pasta.pasta_cpals_coo(x, U, max_iters=1, tol=0.0)
torch.cuda.synchronize(); t = time.perf_counter()
lam, fits, it = pasta.pasta_cpals_coo(x, U, max_iters=iters, tol=0.0)
torch.cuda.synchronize(); print("ms/sweep", (time.perf_counter() - t) * 1e3 / it, fits)
