"""Plain fp64 CPU oracle for the PASTA MTTKRP hot path (ctypes wrapper over oracle.c).

TEST INFRASTRUCTURE ONLY: only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product package ``paper_conf_iiswc_lilwlob20_b200`` never imports it
and shares no code with it.

Each function cites the paper passage it follows (``P:N`` = line N of PAPER.md);
the arithmetic lives in ``oracle.c``.  Inputs are numpy arrays: ``inds`` is a
``uint32`` array of shape ``[N, M]``, ``vals`` a ``float32`` array ``[M]``,
factors a list of ``float32`` arrays ``[I_k, R]`` (row-major).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")

_u32p = C.POINTER(C.c_uint32)
_u64p = C.POINTER(C.c_uint64)
_f32p = C.POINTER(C.c_float)
_f64p = C.POINTER(C.c_double)
_u8p = C.POINTER(C.c_uint8)


def build(force: bool = False) -> str:
    """Compile oracle.c into liboracle.so (gcc, -ffp-contract=off)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fPIC", "-shared",
                               "-o", _SO, _SRC, "-lm"])
    return _SO


_lib = None


def _L():
    global _lib
    if _lib is None:
        build()
        lib = C.CDLL(_SO)
        lib.oracle_mttkrp.restype = C.c_int
        lib.oracle_mttkrp.argtypes = [C.c_uint32, _u32p, C.c_uint64, C.POINTER(_u32p), _f32p,
                                      C.c_uint32, C.POINTER(_f32p), C.c_uint32, _f64p, _f64p]
        lib.oracle_mttkrp_rows.restype = C.c_int
        lib.oracle_mttkrp_rows.argtypes = [C.c_uint32, _u32p, C.c_uint64, C.POINTER(_u32p), _f32p,
                                           C.c_uint32, C.POINTER(_f32p), C.c_uint32, C.c_uint32,
                                           _u32p, _f64p, _f64p]
        lib.oracle_mttkrp_hicoo.restype = C.c_int
        lib.oracle_mttkrp_hicoo.argtypes = [C.c_uint32, _u32p, C.c_uint32, C.c_uint64, _u64p,
                                            C.POINTER(_u32p), C.POINTER(_u8p), _f32p, C.c_uint32,
                                            C.POINTER(_f32p), C.c_uint32, _f64p, _f64p]
        lib.oracle_mode_sort.restype = C.c_int
        lib.oracle_mode_sort.argtypes = [C.c_uint32, C.c_uint64, C.POINTER(_u32p), _f32p,
                                         C.c_uint32, C.POINTER(_u32p), _f32p]
        lib.oracle_coo_to_hicoo.restype = C.c_int64
        lib.oracle_coo_to_hicoo.argtypes = [C.c_uint32, C.c_uint64, C.POINTER(_u32p), _f32p,
                                            C.c_uint32, _u64p, C.POINTER(_u32p), C.POINTER(_u8p),
                                            _f32p]
        lib.oracle_coo_to_ghicoo.restype = C.c_int64
        lib.oracle_coo_to_ghicoo.argtypes = [C.c_uint32, C.c_uint64, C.POINTER(_u32p), _f32p,
                                             C.c_uint32, C.c_uint32, _u64p, C.POINTER(_u32p),
                                             C.POINTER(_u8p), C.POINTER(_u32p), _f32p]
        lib.oracle_mttkrp_ghicoo.restype = C.c_int
        lib.oracle_mttkrp_ghicoo.argtypes = [C.c_uint32, _u32p, C.c_uint32, C.c_uint32, C.c_uint64,
                                             _u64p, C.POINTER(_u32p), C.POINTER(_u8p),
                                             C.POINTER(_u32p), _f32p, C.c_uint32,
                                             C.POINTER(_f32p), C.c_uint32, _f64p, _f64p]
        lib.oracle_gen_slice_powerlaw.restype = C.c_int
        lib.oracle_gen_slice_powerlaw.argtypes = [C.c_uint32, _u32p, C.c_uint64, C.c_uint64,
                                                  C.c_double, C.c_float, C.c_float,
                                                  C.POINTER(_u32p), _f32p]
        lib.oracle_ts.restype = C.c_int
        lib.oracle_ts.argtypes = [C.c_uint64, _f32p, C.c_uint32, C.c_float, _f32p]
        lib.oracle_tew_same.restype = C.c_int
        lib.oracle_tew_same.argtypes = [C.c_uint64, _f32p, _f32p, C.c_uint32, _f32p]
        lib.oracle_tew_merge.restype = C.c_int64
        lib.oracle_tew_merge.argtypes = [C.c_uint32, C.c_uint64, C.POINTER(_u32p), _f32p, C.c_uint64,
                                         C.POINTER(_u32p), _f32p, C.c_uint32, C.POINTER(_u32p), _f32p]
        lib.oracle_ttm.restype = C.c_int64
        lib.oracle_ttm.argtypes = [C.c_uint32, _u32p, C.c_uint64, C.POINTER(_u32p), _f32p, C.c_uint32,
                                   _f32p, C.c_uint32, C.POINTER(_u32p), _f64p, _f64p]
        lib.oracle_relabel.restype = C.c_int
        lib.oracle_relabel.argtypes = [C.c_uint32, _u32p, C.c_uint64, C.c_uint64, C.POINTER(_u32p)]
        lib.oracle_relabel_index.restype = C.c_uint32
        lib.oracle_relabel_index.argtypes = [C.c_uint32, C.c_uint32, C.c_uint64, C.c_uint32]
        lib.oracle_gen_powerlaw.restype = C.c_int
        lib.oracle_gen_powerlaw.argtypes = [C.c_uint32, _u32p, C.c_uint64, C.c_uint64, _f64p,
                                            C.c_double, C.c_float, C.c_float, C.POINTER(_u32p),
                                            _f32p]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray, t):
    return a.ctypes.data_as(t)


def _ptr_list(arrs, t):
    return (t * len(arrs))(*[_ptr(a, t) for a in arrs])


def _prep(dims, inds, vals):
    dims = np.ascontiguousarray(dims, dtype=np.uint32)
    inds = np.ascontiguousarray(inds, dtype=np.uint32)
    vals = np.ascontiguousarray(vals, dtype=np.float32)
    assert inds.ndim == 2 and inds.shape[0] == dims.shape[0] and inds.shape[1] == vals.shape[0]
    return dims, inds, vals


def _factor_list(order, mode, factors, R):
    fl = []
    for k in range(order):
        f = factors[k] if k < len(factors) else None
        if f is None or k == mode:
            f = np.zeros((1, R), np.float32)  # U^(n) is never read (Eq. 3)
        f = np.ascontiguousarray(f, dtype=np.float32)
        assert f.shape[1] == R
        fl.append(f)
    return fl


def mttkrp(dims, inds, vals, mode, factors, R=None):
    """O-MTTKRP, Eq. 3 over nonzeros.  Returns (Mref, Aref) float64 [I_n, R]:
    the result and the per-element sum of |terms| used by the parity tolerance."""
    dims, inds, vals = _prep(dims, inds, vals)
    order = dims.shape[0]
    if R is None:
        R = next(f.shape[1] for k, f in enumerate(factors) if k != mode and f is not None)
    fl = _factor_list(order, mode, factors, R)
    Mref = np.zeros((int(dims[mode]), R), np.float64)
    Aref = np.zeros_like(Mref)
    rows = [np.ascontiguousarray(inds[k]) for k in range(order)]
    rc = _L().oracle_mttkrp(order, _ptr(dims, _u32p), vals.shape[0], _ptr_list(rows, _u32p),
                            _ptr(vals, _f32p), mode, _ptr_list(fl, _f32p), R,
                            _ptr(Mref, _f64p), _ptr(Aref, _f64p))
    if rc != 0:
        raise ValueError("oracle_mttkrp: invalid arguments")
    return Mref, Aref


def mttkrp_rows(dims, inds, vals, mode, factors, rows, R=None):
    """O-MTTKRP restricted to the given output rows (strictly increasing)."""
    dims, inds, vals = _prep(dims, inds, vals)
    order = dims.shape[0]
    if R is None:
        R = next(f.shape[1] for k, f in enumerate(factors) if k != mode and f is not None)
    fl = _factor_list(order, mode, factors, R)
    rows_a = np.ascontiguousarray(rows, dtype=np.uint32)
    assert np.all(np.diff(rows_a.astype(np.int64)) > 0)
    Mref = np.zeros((rows_a.shape[0], R), np.float64)
    Aref = np.zeros_like(Mref)
    irows = [np.ascontiguousarray(inds[k]) for k in range(order)]
    rc = _L().oracle_mttkrp_rows(order, _ptr(dims, _u32p), vals.shape[0],
                                 _ptr_list(irows, _u32p), _ptr(vals, _f32p), mode,
                                 _ptr_list(fl, _f32p), R, rows_a.shape[0], _ptr(rows_a, _u32p),
                                 _ptr(Mref, _f64p), _ptr(Aref, _f64p))
    if rc != 0:
        raise ValueError("oracle_mttkrp_rows: invalid arguments")
    return Mref, Aref


def mttkrp_hicoo(dims, h, mode, factors, R=None):
    """O-HiCOO-MTTKRP (Alg. 3) on a dict from :func:`coo_to_hicoo`."""
    dims = np.ascontiguousarray(dims, dtype=np.uint32)
    order = dims.shape[0]
    if R is None:
        R = next(f.shape[1] for k, f in enumerate(factors) if k != mode and f is not None)
    fl = _factor_list(order, mode, factors, R)
    Mref = np.zeros((int(dims[mode]), R), np.float64)
    Aref = np.zeros_like(Mref)
    binds = [np.ascontiguousarray(h["binds"][k]) for k in range(order)]
    einds = [np.ascontiguousarray(h["einds"][k]) for k in range(order)]
    bptr = np.ascontiguousarray(h["bptr"], dtype=np.uint64)
    vals = np.ascontiguousarray(h["vals"], dtype=np.float32)
    rc = _L().oracle_mttkrp_hicoo(order, _ptr(dims, _u32p), h["block_bits"], h["nblocks"],
                                  _ptr(bptr, _u64p), _ptr_list(binds, _u32p),
                                  _ptr_list(einds, _u8p), _ptr(vals, _f32p), mode,
                                  _ptr_list(fl, _f32p), R, _ptr(Mref, _f64p), _ptr(Aref, _f64p))
    if rc != 0:
        raise ValueError("oracle_mttkrp_hicoo: invalid arguments")
    return Mref, Aref


def mode_sort(inds, vals, mode):
    """O-mode-sort: lexicographic on (i_n, i_{n+1}, ..., i_{n-1}), stable."""
    inds = np.ascontiguousarray(inds, dtype=np.uint32)
    vals = np.ascontiguousarray(vals, dtype=np.float32)
    order, M = inds.shape
    rows = [np.ascontiguousarray(inds[k]) for k in range(order)]
    out = np.empty_like(inds)
    outs = [np.zeros(M, np.uint32) for _ in range(order)]
    ov = np.empty_like(vals)
    rc = _L().oracle_mode_sort(order, M, _ptr_list(rows, _u32p), _ptr(vals, _f32p), mode,
                               _ptr_list(outs, _u32p), _ptr(ov, _f32p))
    if rc != 0:
        raise ValueError("oracle_mode_sort: invalid arguments")
    for k in range(order):
        out[k] = outs[k]
    return out, ov


def coo_to_hicoo(inds, vals, block_bits=7):
    """O-HiCOO conversion (Morton order R#13).  Returns a dict with
    ``bptr`` u64[n_b+1], ``binds`` u32[N][n_b], ``einds`` u8[N][M], ``vals`` f32[M]."""
    inds = np.ascontiguousarray(inds, dtype=np.uint32)
    vals = np.ascontiguousarray(vals, dtype=np.float32)
    order, M = inds.shape
    rows = [np.ascontiguousarray(inds[k]) for k in range(order)]
    bptr = np.zeros(M + 1, np.uint64)
    binds = [np.zeros(max(M, 1), np.uint32) for _ in range(order)]
    einds = [np.zeros(max(M, 1), np.uint8) for _ in range(order)]
    ov = np.zeros(max(M, 1), np.float32)
    nb = _L().oracle_coo_to_hicoo(order, M, _ptr_list(rows, _u32p), _ptr(vals, _f32p), block_bits,
                                  _ptr(bptr, _u64p), _ptr_list(binds, _u32p),
                                  _ptr_list(einds, _u8p), _ptr(ov, _f32p))
    if nb < 0:
        raise ValueError("oracle_coo_to_hicoo: invalid arguments")
    return {
        "order": order, "block_bits": block_bits, "nblocks": int(nb), "nnz": M,
        "bptr": bptr[: nb + 1].copy(),
        "binds": np.stack([b[:nb] for b in binds]) if order else None,
        "einds": np.stack([e[:M] for e in einds]),
        "vals": ov[:M].copy(),
    }


def coo_to_ghicoo(inds, vals, block_bits, cmask):
    """O-gHiCOO conversion (Fig. 2(b); R#29): modes with bit k of ``cmask`` set are
    blocked as in HiCOO, the others stay COO.  Returns a dict with ``bptr`` u64[n_b+1],
    ``binds`` / ``einds`` (lists, None for uncompressed modes), ``uinds`` (list, None for
    compressed modes), ``vals``."""
    inds = np.ascontiguousarray(inds, dtype=np.uint32)
    vals = np.ascontiguousarray(vals, dtype=np.float32)
    order, M = inds.shape
    rows = [np.ascontiguousarray(inds[k]) for k in range(order)]
    bptr = np.zeros(M + 1, np.uint64)
    binds = [np.zeros(max(M, 1), np.uint32) for _ in range(order)]
    einds = [np.zeros(max(M, 1), np.uint8) for _ in range(order)]
    uinds = [np.zeros(max(M, 1), np.uint32) for _ in range(order)]
    ov = np.zeros(max(M, 1), np.float32)
    nb = _L().oracle_coo_to_ghicoo(order, M, _ptr_list(rows, _u32p), _ptr(vals, _f32p),
                                   block_bits, cmask, _ptr(bptr, _u64p), _ptr_list(binds, _u32p),
                                   _ptr_list(einds, _u8p), _ptr_list(uinds, _u32p),
                                   _ptr(ov, _f32p))
    if nb < 0:
        raise ValueError("oracle_coo_to_ghicoo: invalid arguments")
    comp = [bool((cmask >> k) & 1) for k in range(order)]
    return {
        "order": order, "block_bits": block_bits, "cmask": cmask, "nblocks": int(nb), "nnz": M,
        "bptr": bptr[: nb + 1].copy(),
        "binds": [binds[k][:nb].copy() if comp[k] else None for k in range(order)],
        "einds": [einds[k][:M].copy() if comp[k] else None for k in range(order)],
        "uinds": [None if comp[k] else uinds[k][:M].copy() for k in range(order)],
        "vals": ov[:M].copy(),
    }


def mttkrp_ghicoo(dims, g, mode, factors, R=None):
    """O-gHiCOO-MTTKRP: Alg. 3 rebasing the compressed modes only (R#29)."""
    dims = np.ascontiguousarray(dims, dtype=np.uint32)
    order = dims.shape[0]
    if R is None:
        R = next(f.shape[1] for k, f in enumerate(factors) if k != mode and f is not None)
    fl = _factor_list(order, mode, factors, R)
    Mref = np.zeros((int(dims[mode]), R), np.float64)
    Aref = np.zeros_like(Mref)
    dummy32 = np.zeros(1, np.uint32)
    dummy8 = np.zeros(1, np.uint8)
    binds = [np.ascontiguousarray(b) if b is not None else dummy32 for b in g["binds"]]
    einds = [np.ascontiguousarray(e) if e is not None else dummy8 for e in g["einds"]]
    uinds = [np.ascontiguousarray(u) if u is not None else dummy32 for u in g["uinds"]]
    bptr = np.ascontiguousarray(g["bptr"], dtype=np.uint64)
    vals = np.ascontiguousarray(g["vals"], dtype=np.float32)
    rc = _L().oracle_mttkrp_ghicoo(order, _ptr(dims, _u32p), g["block_bits"], g["cmask"],
                                   g["nblocks"], _ptr(bptr, _u64p), _ptr_list(binds, _u32p),
                                   _ptr_list(einds, _u8p), _ptr_list(uinds, _u32p),
                                   _ptr(vals, _f32p), mode, _ptr_list(fl, _f32p), R,
                                   _ptr(Mref, _f64p), _ptr(Aref, _f64p))
    if rc != 0:
        raise ValueError("oracle_mttkrp_ghicoo: invalid arguments")
    return Mref, Aref


def relabel_index(v, dim, seed, k):
    """pi_k(v): the label permutation of mode k (R#22, oracle.c)."""
    return int(_L().oracle_relabel_index(int(v), int(dim), int(seed), int(k)))


def relabel(dims, inds, vals, seed):
    """permute = 1 (R#22): every mode relabelled by pi_k, then the nonzeros re-sorted
    lexicographically (numpy lexsort; coordinates stay distinct, so the order is unique)."""
    dims = np.ascontiguousarray(dims, dtype=np.uint32)
    out = np.ascontiguousarray(inds, dtype=np.uint32).copy()
    rows = [out[k] for k in range(out.shape[0])]
    rc = _L().oracle_relabel(out.shape[0], _ptr(dims, _u32p), out.shape[1], seed, _ptr_list(rows, _u32p))
    if rc != 0:
        raise ValueError("oracle_relabel failed")
    order = np.lexsort(out[::-1])
    return np.ascontiguousarray(out[:, order]), np.ascontiguousarray(vals[order])


def gen_powerlaw(dims, nnz, seed, initiator=None, q=0.75, val_lo=-1.0, val_hi=1.0, permute=False):
    """Stochastic Kronecker generator (R#19-R#23), counter-based.
    Returns (inds u32[N][M] lexicographically sorted, vals f32[M]).  permute: the labels of
    every mode relabelled by pi_k after the draws (R#22), then re-sorted."""
    dims = np.ascontiguousarray(dims, dtype=np.uint32)
    order = dims.shape[0]
    outs = [np.zeros(max(nnz, 1), np.uint32) for _ in range(order)]
    ov = np.zeros(max(nnz, 1), np.float32)
    init_p = None
    if initiator is not None:
        init = np.ascontiguousarray(initiator, dtype=np.float64)
        assert init.shape == (1 << order,)
        init_p = _ptr(init, _f64p)
    rc = _L().oracle_gen_powerlaw(order, _ptr(dims, _u32p), nnz, seed, init_p, q, val_lo, val_hi,
                                  _ptr_list(outs, _u32p), _ptr(ov, _f32p))
    if rc != 0:
        raise ValueError(f"oracle_gen_powerlaw failed rc={rc}")
    inds, vals = np.stack([o[:nnz] for o in outs]), ov[:nnz].copy()
    if permute:
        return relabel(dims, inds, vals, seed)
    return inds, vals


def gen_slice_powerlaw(dims, nnz, seed, alpha=1.0, val_lo=-1.0, val_hi=1.0):
    """FireHose-style slice power-law generator (R#30): every mode index drawn
    independently from P(i) ~ (i+1)^-alpha.  Returns (inds u32[N][M] lexicographic, vals)."""
    dims = np.ascontiguousarray(dims, dtype=np.uint32)
    order = dims.shape[0]
    outs = [np.zeros(max(nnz, 1), np.uint32) for _ in range(order)]
    ov = np.zeros(max(nnz, 1), np.float32)
    rc = _L().oracle_gen_slice_powerlaw(order, _ptr(dims, _u32p), nnz, seed, alpha, val_lo, val_hi,
                                        _ptr_list(outs, _u32p), _ptr(ov, _f32p))
    if rc != 0:
        raise ValueError(f"oracle_gen_slice_powerlaw failed rc={rc}")
    return np.stack([o[:nnz] for o in outs]), ov[:nnz].copy()


def ttm(dims, inds, vals, mode, U):
    """O-TTM (Eq. 2): semi-sparse result over the mode-n fibers of X.
    Returns (fiber_inds u32[N][F] with row `mode` zero, Y f64[F, R], sum|terms| f64[F, R])."""
    dims, inds, vals = _prep(dims, inds, vals)
    order, M = inds.shape
    U = np.ascontiguousarray(U, dtype=np.float32)
    if U.ndim == 1:
        U = U.reshape(-1, 1)
    R = U.shape[1]
    rows = [np.ascontiguousarray(inds[k]) for k in range(order)]
    fib = [np.zeros(max(M, 1), np.uint32) for _ in range(order)]
    y = np.zeros((max(M, 1), R), np.float64)
    ya = np.zeros_like(y)
    nf = _L().oracle_ttm(order, _ptr(dims, _u32p), M, _ptr_list(rows, _u32p), _ptr(vals, _f32p), mode,
                         _ptr(U, _f32p), R, _ptr_list(fib, _u32p), _ptr(y, _f64p), _ptr(ya, _f64p))
    if nf < 0:
        raise ValueError("oracle_ttm: invalid arguments")
    return np.stack([f[:nf] for f in fib]), y[:nf].copy(), ya[:nf].copy()


def ttv(dims, inds, vals, mode, v):
    """O-TTV (Eq. 1): TTM with a single column u = v."""
    f, y, ya = ttm(dims, inds, vals, mode, np.asarray(v, np.float32).reshape(-1, 1))
    return f, y[:, 0].copy(), ya[:, 0].copy()


OPS = {"add": 0, "sub": 1, "mul": 2, "div": 3}


def ts(vals, op, s):
    """O-TS: vals op s, each result rounded once to fp32."""
    vals = np.ascontiguousarray(vals, dtype=np.float32)
    out = np.empty_like(vals)
    if _L().oracle_ts(vals.shape[0], _ptr(vals, _f32p), OPS[op], float(s), _ptr(out, _f32p)) != 0:
        raise ValueError("oracle_ts: invalid arguments")
    return out


def tew_same(a, b, op):
    """O-TEW for identical patterns: a op b element by element."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    b = np.ascontiguousarray(b, dtype=np.float32)
    assert a.shape == b.shape
    out = np.empty_like(a)
    if _L().oracle_tew_same(a.shape[0], _ptr(a, _f32p), _ptr(b, _f32p), OPS[op], _ptr(out, _f32p)) != 0:
        raise ValueError("oracle_tew_same: invalid arguments")
    return out


def tew_merge(ix, vx, iy, vy, op):
    """O-TEW for different patterns (R#31): union (add/sub) or intersection (mul/div),
    lexicographic output.  Returns (inds u32[N][nz], vals f32[nz])."""
    ix = np.ascontiguousarray(ix, dtype=np.uint32)
    iy = np.ascontiguousarray(iy, dtype=np.uint32)
    vx = np.ascontiguousarray(vx, dtype=np.float32)
    vy = np.ascontiguousarray(vy, dtype=np.float32)
    order = ix.shape[0]
    T = vx.shape[0] + vy.shape[0]
    rx = [np.ascontiguousarray(ix[k]) for k in range(order)]
    ry = [np.ascontiguousarray(iy[k]) for k in range(order)]
    outs = [np.zeros(max(T, 1), np.uint32) for _ in range(order)]
    ov = np.zeros(max(T, 1), np.float32)
    nz = _L().oracle_tew_merge(order, vx.shape[0], _ptr_list(rx, _u32p), _ptr(vx, _f32p), vy.shape[0],
                               _ptr_list(ry, _u32p), _ptr(vy, _f32p), OPS[op],
                               _ptr_list(outs, _u32p), _ptr(ov, _f32p))
    if nz == -4:
        raise ValueError("oracle_tew_merge: repeated coordinate inside one input")
    if nz < 0:
        raise ValueError("oracle_tew_merge: invalid arguments")
    return np.stack([o[:nz] for o in outs]), ov[:nz].copy()
