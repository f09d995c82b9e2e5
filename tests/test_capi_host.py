"""CPU-only checks of the C ABI boundary: the library loads, exports every symbol that
include/pasta.h declares, and its host-side logic (argument validation before any side
effect, file parsing errors, the row partitioner) behaves as documented.  No compute call
is made here (there is no GPU on the build box)."""
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "pasta.h")


def _header_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(pasta_[a-z_0-9]+)\s*\(", text)))


@pytest.fixture(scope="module")
def pasta():
    import paper_conf_iiswc_lilwlob20_b200 as p
    from paper_conf_iiswc_lilwlob20_b200 import _native
    if not os.path.exists(_native.LIB_PATH):
        subprocess.check_call(["make", "-C", ROOT, "-j8"], stdout=subprocess.DEVNULL)
    return p


def test_library_exports_every_header_symbol(pasta):
    from paper_conf_iiswc_lilwlob20_b200 import _native
    funcs = _header_functions()
    assert len(funcs) >= 25
    out = subprocess.check_output(["nm", "-D", "--defined-only", _native.LIB_PATH], text=True)
    exported = {line.split()[-1] for line in out.splitlines() if " T " in line}
    missing = [f for f in funcs if f not in exported]
    assert not missing, missing
    # and the ctypes binding declares each of them with the same name
    assert set(funcs) == set(_native.SIGNATURES)
    lib = _native.lib()
    for f in funcs:
        assert hasattr(lib, f)
    assert "sm_100a" in pasta.pasta_version()


def test_validation_happens_before_side_effects(pasta, tmp_path):
    P = pasta
    with pytest.raises(P.PastaError) as e:
        P.pasta_coo_from_arrays([], np.zeros((0, 0), np.uint32), np.zeros(0, np.float32))
    assert e.value.code == -1
    with pytest.raises(P.PastaError) as e:  # index >= dim
        P.pasta_coo_from_arrays([3, 3], np.array([[0, 3], [1, 1]], np.uint32),
                                np.ones(2, np.float32))
    assert e.value.code == -4 and "dims[0]" in str(e.value)
    with pytest.raises(P.PastaError) as e:
        P.pasta_gen_powerlaw([10, 10], 5, seed=1, kind=2, alpha=9.0)
    assert e.value.code == -1
    with pytest.raises(P.PastaError) as e:
        P.pasta_gen_powerlaw([10, 10], 5, seed=1, kind=3)
    assert e.value.code == -1
    with pytest.raises(P.PastaError) as e:
        P.pasta_gen_powerlaw([10, (1 << 27) + 1], 5, seed=1, kind=2)
    assert e.value.code == -4
    with pytest.raises(P.PastaError) as e:
        P.pasta_gen_powerlaw([2, 2], 5, seed=1)
    assert e.value.code == -1
    with pytest.raises(P.PastaError) as e:
        P.pasta_gen_powerlaw([10, 10], 5, seed=1, permute=2)
    assert e.value.code == -1
    with pytest.raises(P.PastaError) as e:
        P.pasta_load_coo(str(tmp_path / "missing.tns"))
    assert e.value.code == -2
    bad = tmp_path / "bad.tns"
    bad.write_text("1 2 3 0.5\n1 2 0.5\n")
    with pytest.raises(P.PastaError) as e:
        P.pasta_load_coo(str(bad))
    assert e.value.code == -3 and "line 2" in str(e.value)
    zero = tmp_path / "zero.tns"
    zero.write_text("# comment\n0 1 1 2.0\n")
    with pytest.raises(P.PastaError) as e:
        P.pasta_load_coo(str(zero))
    assert e.value.code == -3 and "1-based" in str(e.value)
    from paper_conf_iiswc_lilwlob20_b200 import _native
    lib = _native.lib()
    assert lib.pasta_mttkrp_coo(None, 0, None, 16, None, None) == -1
    assert b"NULL" in lib.pasta_last_error()
    assert lib.pasta_profile_read(7, None, None, 0) == -1
    lib.pasta_coo_free(None)  # NULL-safe
    lib.pasta_hicoo_free(None)


def _check_partition(counts, P, bounds):
    n = counts.shape[0]
    assert bounds[0] == 0 and bounds[-1] == n and np.all(np.diff(bounds.astype(np.int64)) >= 0)
    T = int(counts.sum())
    S = np.concatenate([[0], np.cumsum(counts.astype(np.int64))])
    for p in range(1, P):
        r = int(bounds[p])
        # minimality: bounds[p] is the first r with S(r) * P >= p * T
        assert S[r] * P >= p * T
        assert r == 0 or S[r - 1] * P < p * T
    part = [int(S[bounds[p + 1]] - S[bounds[p]]) for p in range(P)]
    assert sum(part) == T
    assert max(part) <= T / P + (counts.max() if n else 0) + 1


@pytest.mark.parametrize("seed", range(4))
def test_row_partition_host_logic(pasta, seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 5000))
    counts = (rng.pareto(1.2, size=n) * 10).astype(np.uint64)
    for P in (1, 2, 3, 8):
        b = pasta.pasta_row_partition(counts, P)
        _check_partition(counts, P, b)


def test_row_partition_edge_cases(pasta):
    # a single heavy row larger than T / P: the imbalance is accepted, ranges stay valid
    counts = np.array([0, 1000, 1, 1], np.uint64)
    b = pasta.pasta_row_partition(counts, 4)
    _check_partition(counts, 4, b)
    # empty tensor
    b = pasta.pasta_row_partition(np.zeros(5, np.uint64), 3)
    assert list(b) == [0, 0, 0, 5]
    with pytest.raises(pasta.PastaError):
        pasta.pasta_row_partition(np.ones(3, np.uint64), 0)


def _pbin(order, nnz, dims, inds, vals, flags=0, extra=b""):
    import struct
    b = b"PASTAB01" + struct.pack("<IIQ", order, flags, nnz) + struct.pack(f"<{order}I", *dims)
    for k in range(order):
        b += np.asarray(inds[k], np.uint32).tobytes()
    return b + np.asarray(vals, np.float32).tobytes() + extra


def test_pbin_header_and_range_errors(pasta, tmp_path):
    """.pbin binary cache (R#17): malformed files are rejected before any upload."""
    P = pasta
    p = tmp_path / "x.pbin"
    inds = [[0, 1], [2, 0]]
    cases = [
        (_pbin(2, 2, (3, 3), inds, [1, 2], extra=b"\0"), -3),   # size != header
        (_pbin(2, 2, (3, 3), inds, [1, 2])[:-3], -3),            # truncated
        (_pbin(9, 2, (3,) * 9, [[0, 0]] * 9, [1, 2]), -3),       # order > 8
        (_pbin(2, 2, (3, 3), inds, [1, 2], flags=1), -3),        # unknown flags
        (_pbin(2, 2, (3, 2), inds, [1, 2]), -4),                 # index 2 >= dims[1]
        (_pbin(2, 2, (0, 3), inds, [1, 2]), -1),                 # a zero dim
    ]
    for blob, code in cases:
        p.write_bytes(blob)
        with pytest.raises(P.PastaError) as e:
            P.pasta_load_coo(str(p))
        assert e.value.code == code, (code, str(e.value))
