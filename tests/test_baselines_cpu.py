"""The optional paper-method CPU baseline (baselines/, COO-MTTKRP-OMP: fp32, omp atomic, all
cores) computes MTTKRP within the north_star tolerance of the oracle."""
import numpy as np

import synth_inputs as si


def test_omp_baseline_matches_oracle(oracle_mod):
    import baselines
    dims = (300, 200, 500)
    inds, vals = si.powerlaw_coo(dims, 50_000, seed=3)
    U = si.factors(dims, 16, seed=1)
    for n in range(3):
        got = baselines.mttkrp(dims, inds, vals, n, U)
        ref, ab = oracle_mod.mttkrp(dims, inds, vals, n, U)
        assert np.all(np.abs(got - ref) <= 1e-4 * ab + 1e-6), n
