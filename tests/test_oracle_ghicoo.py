"""Pins of the oracle's COO -> gHiCOO conversion and gHiCOO-MTTKRP (CPU only).

gHiCOO (Fig. 2(b)): "pick which modes to be compressed in units of blocks for
HiCOO and which stay in COO format".  Reading R#29: order = Morton order (R#13) of the
compressed modes' coordinates, ties lexicographic over the uncompressed modes.

Pins that do not re-run the oracle's own code:
* an independent pure-Python conversion that builds the interleaved bit string of the
  compressed modes explicitly and sorts by (bits, uncompressed coordinates, position);
* the special cases that reduce to other routines: cmask = all modes is HiCOO (the
  oracle's HiCOO is itself pinned by the Python Morton reference in test_oracle_hicoo),
  cmask = {0} is the mode-0 lexicographic sort (numpy lexsort);
* n_b = number of distinct compressed block keys (numpy unique), round trip, storage
  formula (Table I P:117 generalised: (N_c + 4N_u + 4) M + (8 + 4 N_c) n_b bytes);
* gHiCOO-MTTKRP equals the brute-force-pinned COO MTTKRP to fp64 rounding.
"""
import numpy as np
import pytest

import synth_inputs as si


def _python_ghicoo(inds, vals, b, cmask):
    N, M = inds.shape
    comp = [k for k in range(N) if (cmask >> k) & 1]
    unc = [k for k in range(N) if not (cmask >> k) & 1]

    def key(x):
        bits = []
        for lvl in range(31, -1, -1):  # MSB level first
            for k in comp:  # lowest compressed mode first within a level
                bits.append((int(inds[k, x]) >> lvl) & 1)
        return (tuple(bits), tuple(int(inds[k, x]) for k in unc), x)

    order = sorted(range(M), key=key)
    bptr, binds = [], {k: [] for k in comp}
    prev = None
    for pos, x in enumerate(order):
        blk = tuple(int(inds[k, x]) >> b for k in comp)
        if blk != prev:
            bptr.append(pos)
            for j, k in enumerate(comp):
                binds[k].append(blk[j])
            prev = blk
    bptr.append(M)
    o = np.array(order, dtype=np.int64)
    return (np.array(bptr, np.uint64), {k: np.array(binds[k], np.uint32) for k in comp},
            {k: (inds[k, o] & ((1 << b) - 1)).astype(np.uint8) for k in comp},
            {k: inds[k, o].astype(np.uint32) for k in unc}, vals[o])


@pytest.mark.parametrize("dims,nnz,b,cmask,seed", [
    ((40, 50, 60), 300, 3, 0b101, 1),
    ((300, 200, 100), 500, 7, 0b001, 2),
    ((300, 200, 100), 500, 4, 0b110, 3),
    ((17, 33, 9, 5), 400, 2, 0b1010, 4),
    ((17, 33, 9, 5), 400, 2, 0b0111, 5),
    ((7, 7), 20, 8, 0b10, 6),
])
def test_conversion_matches_independent_python(oracle_mod, dims, nnz, b, cmask, seed):
    inds, vals = si.powerlaw_coo(dims, nnz, seed=seed)
    g = oracle_mod.coo_to_ghicoo(inds, vals, b, cmask)
    bptr, binds, einds, uinds, v = _python_ghicoo(inds, vals, b, cmask)
    assert g["nblocks"] == len(bptr) - 1
    np.testing.assert_array_equal(g["bptr"], bptr)
    for k in range(len(dims)):
        if (cmask >> k) & 1:
            np.testing.assert_array_equal(g["binds"][k], binds[k])
            np.testing.assert_array_equal(g["einds"][k], einds[k])
            assert g["uinds"][k] is None
        else:
            np.testing.assert_array_equal(g["uinds"][k], uinds[k])
            assert g["binds"][k] is None and g["einds"][k] is None
    np.testing.assert_array_equal(g["vals"].view(np.uint32), v.view(np.uint32))


@pytest.mark.parametrize("dims,b", [((300, 200, 100), 5), ((17, 33, 9, 5), 2)])
def test_all_modes_is_hicoo(oracle_mod, dims, b):
    inds, vals = si.powerlaw_coo(dims, 600, seed=11)
    N = len(dims)
    g = oracle_mod.coo_to_ghicoo(inds, vals, b, (1 << N) - 1)
    h = oracle_mod.coo_to_hicoo(inds, vals, b)
    assert g["nblocks"] == h["nblocks"]
    np.testing.assert_array_equal(g["bptr"], h["bptr"])
    for k in range(N):
        np.testing.assert_array_equal(g["binds"][k], h["binds"][k])
        np.testing.assert_array_equal(g["einds"][k], h["einds"][k])
    np.testing.assert_array_equal(g["vals"].view(np.uint32), h["vals"].view(np.uint32))


def test_mode0_only_is_lexicographic(oracle_mod):
    dims = (1000, 300, 200)
    inds, vals = si.powerlaw_coo(dims, 3000, seed=12)
    b = 5
    g = oracle_mod.coo_to_ghicoo(inds, vals, b, 0b001)
    o = np.lexsort(inds[::-1])  # mode 0 primary, then 1, then 2 (numpy, independent)
    full0 = (np.repeat(g["binds"][0], np.diff(g["bptr"].astype(np.int64))).astype(np.uint32) << b) \
        + g["einds"][0]
    np.testing.assert_array_equal(full0, inds[0, o])
    np.testing.assert_array_equal(g["uinds"][1], inds[1, o])
    np.testing.assert_array_equal(g["uinds"][2], inds[2, o])
    np.testing.assert_array_equal(g["vals"], vals[o])
    # blocks = distinct i_0 >> b, in increasing order
    np.testing.assert_array_equal(g["binds"][0], np.unique(inds[0] >> b))


@pytest.mark.parametrize("cmask", [0b001, 0b010, 0b100, 0b011, 0b101, 0b110, 0b111])
def test_structure_storage_roundtrip(oracle_mod, cmask):
    dims = (320, 28000, 1600)
    inds, vals = si.powerlaw_coo(dims, 5000, seed=13)
    b, N, M = 7, 3, 5000
    g = oracle_mod.coo_to_ghicoo(inds, vals, b, cmask)
    comp = [k for k in range(N) if (cmask >> k) & 1]
    nb = g["nblocks"]
    keys = np.stack([inds[k] >> b for k in comp], axis=1)
    assert nb == np.unique(keys, axis=0).shape[0]
    bptr = g["bptr"].astype(np.int64)
    assert bptr[0] == 0 and bptr[-1] == M and np.all(np.diff(bptr) > 0)
    full = np.zeros((N, M), np.int64)
    blk = np.repeat(np.arange(nb), np.diff(bptr))
    for k in range(N):
        if k in comp:
            full[k] = g["binds"][k].astype(np.int64)[blk] * (1 << b) + g["einds"][k]
        else:
            full[k] = g["uinds"][k]
    rec = sorted(zip(*[full[k] for k in range(N)], g["vals"].tolist()))
    orig = sorted(zip(*[inds[k].astype(np.int64) for k in range(N)], vals.tolist()))
    assert rec == orig
    nc, nu = len(comp), N - len(comp)
    nbytes = (sum(g["einds"][k].nbytes + g["binds"][k].nbytes for k in comp)
              + sum(g["uinds"][k].nbytes for k in range(N) if k not in comp)
              + g["vals"].nbytes + g["bptr"].nbytes - 8)
    assert nbytes == (nc + 4 * nu + 4) * M + (8 + 4 * nc) * nb


def test_invalid_masks(oracle_mod):
    inds, vals = si.uniform_coo((10, 10, 10), 20, seed=1)
    for bad in (0, 0b1000):
        with pytest.raises(ValueError):
            oracle_mod.coo_to_ghicoo(inds, vals, 3, bad)


@pytest.mark.parametrize("dims,b,cmask", [((40, 50, 60), 3, 0b101), ((300, 200, 100, 20), 5, 0b0011),
                                          ((300, 200, 100, 20), 5, 0b1000)])
def test_ghicoo_mttkrp_equals_coo_mttkrp(oracle_mod, dims, b, cmask):
    inds, vals = si.powerlaw_coo(dims, 2000, seed=5)
    U = si.factors(dims, 6, seed=1)
    g = oracle_mod.coo_to_ghicoo(inds, vals, b, cmask)
    for n in range(len(dims)):
        a, aa = oracle_mod.mttkrp(dims, inds, vals, n, U)
        c, ca = oracle_mod.mttkrp_ghicoo(dims, g, n, U)
        np.testing.assert_allclose(c, a, rtol=1e-12, atol=1e-12 * (1 + aa.max()))
        np.testing.assert_allclose(ca, aa, rtol=1e-12, atol=1e-12)
