"""Plain CP-ALS oracle (TEST INFRASTRUCTURE ONLY, like the rest of oracle/).

CANDECOMP/PARAFAC by alternating least squares, the decomposition whose bottleneck is
MTTKRP (CPD is the paper's future work).  The update is the textbook one of the
paper's ref. [1] (Kolda & Bader), written out step by step in fp64 with numpy, with the
oracle's own MTTKRP (oracle.mttkrp, Eq. 3):

    for each sweep, for n = 0..N-1:
        M   = X_(n) (KRP_{k != n} U_k)            -- oracle.mttkrp
        V   = Hadamard_{k != n} (U_k^T U_k)
        U_n = M V^{-1}                             -- np.linalg.solve
        lambda_r = ||U_n(:, r)||_2;  U_n(:, r) /= lambda_r
    fit = 1 - ||X - [[lambda; U]]||_F / ||X||_F,
        ||X - Xhat||^2 = ||X||^2 + lambda^T (Hadamard_k U_k^T U_k) lambda - 2 <X, Xhat>,
        <X, Xhat> = sum_{i,r} lambda_r M(i, r) U_last(i, r)   (M of the last mode)

Factors are stored in fp32 between updates (the storage precision of the GPU path and the
input type of oracle.mttkrp); every arithmetic step is fp64.  Pinned in
tests/test_oracle_cpals.py by exact recovery of a rank-R tensor, the normal equations, a
brute-force dense fit and ALS monotonicity.
"""
from __future__ import annotations

import numpy as np

from . import mttkrp


def cp_als(dims, inds, vals, U0, iters, tol=0.0, record=None, perturb=None):
    """Run `iters` sweeps (or stop when |fit - previous| < tol after the first sweep).
    U0: list of float32 [I_k, R] initial factors.  Returns (U list fp32, lambda fp64, fits).
    perturb (test hook, default None = the plain algorithm): perturb(stage, n, array) -> array
    applied to M ("M", with the oracle's sum|terms| as array.A), to each gram U_k^T U_k ("G")
    and to the solved factor before normalisation ("U"); used to measure the algorithm's
    sensitivity to the rounding of an fp32 implementation (R#33)."""
    N = len(dims)
    U = [np.ascontiguousarray(u, dtype=np.float32) for u in U0]
    R = U[0].shape[1]
    lam = np.ones(R)
    normx2 = float(np.sum(np.asarray(vals, np.float64) ** 2))
    fits = []
    M = None
    for it in range(iters):
        for n in range(N):
            M, A = mttkrp(dims, inds, vals, n, U, R=R)
            if perturb is not None:
                M = perturb("M", n, (M, A))
            V = np.ones((R, R))
            for k in range(N):
                if k != n:
                    Uk = U[k].astype(np.float64)
                    Gk = Uk.T @ Uk
                    V *= perturb("G", k, (Gk, np.abs(Uk).T @ np.abs(Uk))) if perturb is not None else Gk
            Un = np.linalg.solve(V.T, M.T).T  # U_n V = M
            if perturb is not None:
                Un = perturb("U", n, (Un, None))
            if record is not None:
                record.append((n, M.copy(), V.copy(), Un.copy()))
            lam = np.sqrt(np.sum(Un * Un, axis=0))
            lam[lam == 0] = 1.0
            U[n] = (Un / lam).astype(np.float32)
        G = np.ones((R, R))
        for k in range(N):
            Uk = U[k].astype(np.float64)
            G *= Uk.T @ Uk
        nxhat2 = float(lam @ G @ lam)
        inner = float(np.sum(lam * np.sum(M * U[N - 1].astype(np.float64), axis=0)))
        resid2 = max(normx2 + nxhat2 - 2.0 * inner, 0.0)
        fit = 1.0 - np.sqrt(resid2) / np.sqrt(normx2) if normx2 > 0 else 0.0
        fits.append(fit)
        if it > 0 and abs(fits[-1] - fits[-2]) < tol:
            break
    return U, lam, fits
