"""Pins of the oracle's COO -> HiCOO conversion and HiCOO-MTTKRP (CPU only).

The Morton order reading (R#13) is pinned by an independent pure-Python
implementation that builds the interleaved bit string explicitly and sorts by
it; the block structure by invariants of P:181/P:205 and the storage formula of
Table I: (N+4) M + (8+4N) n_b bytes, 7M + 20 n_b at N = 3.
"""
import numpy as np
import pytest

import synth_inputs as si


def _python_hicoo(inds, vals, b):
    N, M = inds.shape
    nbits = 32

    def key(x):
        bits = []
        for lvl in range(nbits - 1, -1, -1):  # MSB level first
            for k in range(N):  # mode 0 first within a level
                bits.append((int(inds[k, x]) >> lvl) & 1)
        return (tuple(bits), x)

    order = sorted(range(M), key=key)
    bptr, binds = [], [[] for _ in range(N)]
    prev = None
    for pos, x in enumerate(order):
        blk = tuple(int(inds[k, x]) >> b for k in range(N))
        if blk != prev:
            bptr.append(pos)
            for k in range(N):
                binds[k].append(blk[k])
            prev = blk
    bptr.append(M)
    einds = np.array([[int(inds[k, x]) & ((1 << b) - 1) for x in order] for k in range(N)],
                     dtype=np.uint8).reshape(N, M)
    return (np.array(bptr, np.uint64), np.array(binds, np.uint32).reshape(N, -1), einds,
            vals[np.array(order, dtype=np.int64)] if M else vals)


@pytest.mark.parametrize("dims,nnz,b,seed", [
    ((40, 50, 60), 300, 3, 1),
    ((300, 200, 100), 500, 7, 2),
    ((17, 33, 9, 5), 400, 2, 3),
    ((1000,), 100, 4, 4),
    ((7, 7), 20, 8, 5),
])
def test_conversion_matches_independent_python(oracle_mod, dims, nnz, b, seed):
    inds, vals = si.powerlaw_coo(dims, nnz, seed=seed)
    h = oracle_mod.coo_to_hicoo(inds, vals, b)
    bptr, binds, einds, v = _python_hicoo(inds, vals, b)
    assert h["nblocks"] == len(bptr) - 1
    np.testing.assert_array_equal(h["bptr"], bptr)
    np.testing.assert_array_equal(h["binds"], binds)
    np.testing.assert_array_equal(h["einds"], einds)
    np.testing.assert_array_equal(h["vals"].view(np.uint32), v.view(np.uint32))


def test_structure_invariants_and_storage(oracle_mod):
    dims = (12092, 9184, 28818)
    inds, vals = si.powerlaw_coo(dims, 20000, seed=7)
    b = 7
    h = oracle_mod.coo_to_hicoo(inds, vals, b)
    nb, M, N = h["nblocks"], vals.shape[0], 3
    bptr = h["bptr"].astype(np.int64)
    assert bptr[0] == 0 and bptr[-1] == M and np.all(np.diff(bptr) > 0)
    assert np.all(h["einds"] < (1 << b))
    # blocks strictly increasing in Morton order of block coordinates, all distinct
    blocks = {tuple(h["binds"][:, j]) for j in range(nb)}
    assert len(blocks) == nb
    # round trip: the multiset of (coords, value) is preserved
    rec = []
    for j in range(nb):
        for x in range(bptr[j], bptr[j + 1]):
            rec.append(tuple(int(h["binds"][k, j]) * (1 << b) + int(h["einds"][k, x])
                             for k in range(N)) + (float(h["vals"][x]),))
    orig = [tuple(int(inds[k, x]) for k in range(N)) + (float(vals[x]),) for x in range(M)]
    assert sorted(rec) == sorted(orig)
    # Table I tensor part at N = 3: 7M + 20 n_b bytes (einds u8, val f32, bptr u64,
    # binds u32); general: (N+4) M + (8+4N) n_b
    nbytes = h["einds"].nbytes + h["vals"].nbytes + (h["bptr"].nbytes - 8) + h["binds"].nbytes
    assert nbytes == 7 * M + 20 * nb == (N + 4) * M + (8 + 4 * N) * nb


def test_edge_cases(oracle_mod):
    # B >= max dim -> one block
    inds, vals = si.uniform_coo((100, 90, 80), 50, seed=3)
    h = oracle_mod.coo_to_hicoo(inds, vals, 7)
    assert h["nblocks"] == 1 and list(h["binds"][:, 0]) == [0, 0, 0]
    # order 1 -> numeric sort
    inds1 = np.array([[900, 5, 300, 7, 128]], np.uint32)
    vals1 = np.arange(5, dtype=np.float32)
    h1 = oracle_mod.coo_to_hicoo(inds1, vals1, 7)
    full = h1["binds"][0][np.searchsorted(h1["bptr"][1:], np.arange(5), side="right")] * 128 \
        + h1["einds"][0]
    np.testing.assert_array_equal(full, [5, 7, 128, 300, 900])
    # empty tensor
    h0 = oracle_mod.coo_to_hicoo(np.zeros((3, 0), np.uint32), np.zeros(0, np.float32), 7)
    assert h0["nblocks"] == 0 and list(h0["bptr"]) == [0]
    # a dim of 1 and dims not multiples of B
    inds2, vals2 = si.uniform_coo((1, 300, 129), 200, seed=9)
    h2 = oracle_mod.coo_to_hicoo(inds2, vals2, 7)
    assert np.all(h2["binds"][0] == 0) and np.all(h2["einds"][0] == 0)


@pytest.mark.parametrize("dims,b", [((40, 50, 60), 3), ((300, 200, 100, 20), 5)])
def test_hicoo_mttkrp_equals_coo_mttkrp(oracle_mod, dims, b):
    inds, vals = si.powerlaw_coo(dims, 2000, seed=5)
    U = si.factors(dims, 6, seed=1)
    h = oracle_mod.coo_to_hicoo(inds, vals, b)
    for n in range(len(dims)):
        a, aa = oracle_mod.mttkrp(dims, inds, vals, n, U)
        c, ca = oracle_mod.mttkrp_hicoo(dims, h, n, U)
        np.testing.assert_allclose(c, a, rtol=1e-12, atol=1e-12 * (1 + aa.max()))
        np.testing.assert_allclose(ca, aa, rtol=1e-12, atol=1e-12)
