"""Seeded synthetic inputs shared by tests, smoke and bench.

This module only draws random tensors and factor matrices; it holds none of the
MTTKRP arithmetic, none of the HiCOO conversion and none of the product
generator.  Both the oracle (``oracle/``) and the CUDA library
(``paper_conf_iiswc_lilwlob20_b200``) receive the SAME arrays from here, so no
oracle input ever comes from the CUDA path.

Recipe ("Input recipe"): coordinates are unique; values U[-1, 1)
float32 (mixed signs exercise the sum-|terms| tolerance); factor entries U[0, 1)
float32, row-major [I_k, R].  ``powerlaw_coo`` draws each mode's index
bits independently with P(bit = 1) = 1 - q (q = 0.75), the product-form
Kronecker distribution of the paper's regular synthetic tensors, and
keeps the first occurrence of repeated coordinates.
"""
from __future__ import annotations

import numpy as np


def _rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.Philox(seed))


def _unique_first(coords: np.ndarray) -> np.ndarray:
    """Indices (in draw order) of the first occurrence of each distinct row of coords [D, N]."""
    D, N = coords.shape
    if D == 0:
        return np.zeros(0, np.int64)
    order = np.lexsort([coords[:, k] for k in range(N - 1, -1, -1)])  # stable, mode 0 primary
    srt = coords[order]
    new = np.ones(D, bool)
    new[1:] = np.any(srt[1:] != srt[:-1], axis=1)
    return np.sort(order[new])


def uniform_coo(dims, nnz, seed, shuffle=True):
    """nnz distinct coordinates uniform over prod(dims); returns (inds u32[N,M], vals f32[M])."""
    dims = [int(d) for d in dims]
    rng = _rng(seed)
    total = int(np.prod(np.array(dims, dtype=np.float64)))
    if nnz > total:
        raise ValueError("nnz > number of cells")
    got = np.zeros((0, len(dims)), np.uint32)
    while got.shape[0] < nnz:
        need = (nnz - got.shape[0]) * 2 + 64
        cand = np.stack([rng.integers(0, d, size=need, dtype=np.uint64) for d in dims], axis=1)
        allc = np.concatenate([got.astype(np.uint64), cand])
        got = allc[_unique_first(allc)].astype(np.uint32)
    got = got[:nnz]
    if not shuffle:
        order = np.lexsort(got.T[::-1])
        got = got[order]
    vals = rng.uniform(-1.0, 1.0, size=nnz).astype(np.float32)
    return np.ascontiguousarray(got.T), vals


def powerlaw_coo(dims, nnz, seed, q=0.75, shuffle=True, dedup=True):
    """Product-form Kronecker power-law tensor (independent index bits, P(1) = 1 - q).
    dedup=False skips the uniqueness pass (full-size inputs where repeats are ~1e-7 of the
    draws); repeated coordinates are then separate nonzeros (R#15)."""
    dims = [int(d) for d in dims]
    rng = _rng(seed)
    L = [max(0, int(np.ceil(np.log2(d)))) if d > 1 else 0 for d in dims]
    got = np.zeros((0, len(dims)), np.uint64)
    while got.shape[0] < nnz:
        need = int((nnz - got.shape[0]) * 1.3) + 1024
        cols = []
        for d, l in zip(dims, L):
            mask = np.uint64((1 << l) - 1)
            if q == 0.75 and l <= 32:
                # AND of two uniform words: every bit is 1 with probability 1/4, independently
                a = rng.integers(0, 1 << 32, size=need, dtype=np.uint32)
                b = rng.integers(0, 1 << 32, size=need, dtype=np.uint32)
                idx = ((a & b).astype(np.uint64)) & mask
            else:
                idx = np.zeros(need, np.uint64)
                for bb in range(l):
                    bit = (rng.random(need) < (1.0 - q)).astype(np.uint64)
                    idx |= bit << np.uint64(bb)
            cols.append(idx)
        cand = np.stack(cols, axis=1)
        ok = np.all(cand < np.array(dims, dtype=np.uint64)[None, :], axis=1)
        allc = np.concatenate([got, cand[ok]])
        got = allc[_unique_first(allc)] if dedup else allc
    got = got[:nnz].astype(np.uint32)
    if shuffle:
        got = got[rng.permutation(nnz)]
    vals = rng.uniform(-1.0, 1.0, size=nnz).astype(np.float32)
    return np.ascontiguousarray(got.T), vals


def powerlaw_coo_lean(dims, nnz, seed, chunk=1 << 24):
    """powerlaw_coo(dedup=False, shuffle=False) for BASELINE-size inputs (C5: 1B nonzeros) in
    bounded memory: every mode must be a power of two (no rejection step); arrays are filled
    chunk by chunk (u32 [N, M] + f32 [M], nothing else of that size).  Bits of mode k are
    1 with probability 1/4 (AND of two uniform words), the q = 0.75 product-form law."""
    dims = [int(d) for d in dims]
    for d in dims:
        if d & (d - 1) or d > (1 << 32):
            raise ValueError("powerlaw_coo_lean needs power-of-two dims")
    rng = _rng(seed)
    inds = np.empty((len(dims), nnz), np.uint32)
    vals = np.empty(nnz, np.float32)
    for lo in range(0, nnz, chunk):
        n = min(chunk, nnz - lo)
        for k, d in enumerate(dims):
            a = rng.integers(0, 1 << 32, size=n, dtype=np.uint32)
            a &= rng.integers(0, 1 << 32, size=n, dtype=np.uint32)
            a &= np.uint32(d - 1)
            inds[k, lo:lo + n] = a
        vals[lo:lo + n] = rng.uniform(-1.0, 1.0, size=n)
    return inds, vals


def factors(dims, R, seed, lo=0.0, hi=1.0):
    """Dense factor matrices U^(k) in R^{I_k x R}, row-major float32, entries U[lo, hi)."""
    rng = _rng(seed + 7919)
    return [rng.uniform(lo, hi, size=(int(d), R)).astype(np.float32) for d in dims]


def hot_row_coo(dims, nnz_hot, nnz_rest, seed, mode=0, hot_row=None):
    """A tensor whose mode-`mode` row `hot_row` holds nnz_hot nonzeros (plus nnz_rest uniform
    ones elsewhere): the power-law worst case for segmented reductions."""
    dims = [int(d) for d in dims]
    rng = _rng(seed)
    hot_row = dims[mode] // 2 if hot_row is None else hot_row
    other = [d for k, d in enumerate(dims) if k != mode]
    total_other = int(np.prod(np.array(other, dtype=np.float64)))
    if nnz_hot > total_other:
        raise ValueError("hot row cannot hold that many distinct nonzeros")
    lin = rng.choice(total_other, size=nnz_hot, replace=False) if total_other < 4 * nnz_hot \
        else np.unique(rng.integers(0, total_other, size=int(nnz_hot * 1.2) + 16))[:nnz_hot]
    while lin.shape[0] < nnz_hot:
        extra = rng.integers(0, total_other, size=nnz_hot)
        lin = np.unique(np.concatenate([lin, extra]))[:nnz_hot]
    lin = rng.permutation(lin)
    cols = []
    rem = lin.astype(np.int64)
    for d in other:
        cols.append((rem % d).astype(np.uint32))
        rem //= d
    hot = []
    j = 0
    for k in range(len(dims)):
        if k == mode:
            hot.append(np.full(nnz_hot, hot_row, np.uint32))
        else:
            hot.append(cols[j]); j += 1
    hot = np.stack(hot)
    if nnz_rest:
        rest, _ = uniform_coo(dims, nnz_rest, seed + 1)
        keep = rest[mode] != hot_row
        rest = rest[:, keep]
        inds = np.concatenate([hot, rest], axis=1)
    else:
        inds = hot
    perm = rng.permutation(inds.shape[1])
    inds = np.ascontiguousarray(inds[:, perm])
    vals = rng.uniform(-1.0, 1.0, size=inds.shape[1]).astype(np.float32)
    return inds, vals


# Shapes of the BASELINE.json configs.
CONFIGS = {
    "c1": dict(name="uniform-100^3", dims=(100, 100, 100), nnz=10_000, R=16, kind="uniform",
               seed=1001),
    "c2": dict(name="nell2-shaped", dims=(12092, 9184, 28818), nnz=77_000_000, R=16,
               kind="powerlaw", seed=1002),
    "c3": dict(name="flickr-shaped", dims=(320_000, 28_000_000, 1_600_000), nnz=113_000_000,
               R=16, kind="powerlaw", seed=1003),
    "c4": dict(name="enron-shaped", dims=(6066, 5699, 244268, 1176), nnz=54_000_000, R=16,
               kind="powerlaw", seed=1004),
    "h": dict(name="regL-shaped-100M", dims=(1 << 23, 1 << 23, 1 << 23), nnz=100_000_000, R=16,
              kind="powerlaw", seed=1006),
    "c5": dict(name="regL-shaped-1B", dims=(1 << 23, 1 << 23, 1 << 23), nnz=1_000_000_000, R=32,
               kind="powerlaw", seed=1005),
}
