"""pasta-b200: B200-native sparse MTTKRP on COO and HiCOO (Li et al., IISWC'20).

Thin Python binding over the C ABI of ``lib/libpasta.so`` (``include/pasta.h``): the
functions carry the C names and only marshal arguments.  Every compute step (generation,
sorting, HiCOO conversion, MTTKRP) runs in the library's CUDA kernels; PyTorch supplies
device memory, streams and process groups.  There is no CPU fallback: importing works
without a GPU, but compute calls raise ``PastaError`` (PASTA_ECUDA) when no device exists.
"""
from __future__ import annotations

import ctypes as C
from typing import Optional, Sequence

import numpy as np

from ._native import MAX_ORDER, Allocator, ALLOC_FN, FREE_FN, GenParams, PastaError, check, lib

__all__ = [
    "PastaError", "Coo", "Hicoo", "pasta_version", "pasta_set_allocator", "use_torch_allocator",
    "pasta_load_coo", "pasta_save_coo", "pasta_coo_from_arrays", "pasta_gen_powerlaw",
    "pasta_coo_to_hicoo", "pasta_coo_prepare", "pasta_coo_release_mode", "pasta_hicoo_prepare", "pasta_mttkrp_coo",
    "pasta_mttkrp_hicoo", "pasta_mttkrp_coo_bcast", "pasta_mttkrp_coo_allmodes_host", "pasta_mttkrp_coo_allmodes_host_batch",
    "pasta_coo_row_counts",
    "pasta_row_partition", "pasta_coo_partition", "pasta_coo_shard", "pasta_hicoo_shard", "pasta_coo_info",
    "pasta_coo_export", "pasta_coo_export_mode", "pasta_hicoo_info", "pasta_hicoo_export",
    "pasta_launch_count", "pasta_die_map", "pasta_profile_enable", "pasta_profile_read", "pasta_gram",
    "pasta_cpals_solve", "pasta_normalize_columns", "pasta_weighted_inner", "pasta_coo_norm2",
    "pasta_cpals_coo", "pasta_coo_fibers", "pasta_coo_fiber_export", "pasta_ttm_coo",
    "pasta_ttv_coo", "pasta_coo_to_ghicoo", "pasta_ghicoo_auto_mask", "pasta_ghicoo_export",
    "pasta_cpals_prepare", "pasta_cpals_fit", "pasta_rows_times", "pasta_rows_times_bcast", "pasta_bcast_f32", "pasta_dev_alloc",
    "pasta_dev_free", "pasta_ipc_get_handle", "pasta_ipc_open", "pasta_ipc_close", "pasta_ts", "pasta_tew", "pasta_coo_values_ptr", "pasta_coo_ts", "pasta_coo_tew", "OPS",
]

_u32p = C.POINTER(C.c_uint32)
_u64p = C.POINTER(C.c_uint64)
_f32p = C.POINTER(C.c_float)
_u8p = C.POINTER(C.c_uint8)


class Coo:
    """Owning wrapper of a ``pasta_coo*`` (device-resident COO tensor)."""

    def __init__(self, ptr: int):
        self._p = C.c_void_p(ptr)
        order, dims, nnz = pasta_coo_info(self)
        self.order, self.dims, self.nnz = order, dims, nnz

    @property
    def ptr(self):
        return self._p

    def free(self):
        if self._p and self._p.value:
            lib().pasta_coo_free(self._p)
            self._p = C.c_void_p(None)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class Hicoo:
    """Owning wrapper of a ``pasta_hicoo*`` (device-resident HiCOO tensor)."""

    def __init__(self, ptr: int):
        self._p = C.c_void_p(ptr)
        info = pasta_hicoo_info(self)
        self.order, self.dims, self.block_bits, self.nblocks, self.nnz = info
        cm = C.c_uint32()
        check(lib().pasta_ghicoo_info(self._p, C.byref(cm)))
        self.cmask = cm.value  # gHiCOO compression mask (all bits: HiCOO)

    @property
    def ptr(self):
        return self._p

    def free(self):
        if self._p and self._p.value:
            lib().pasta_hicoo_free(self._p)
            self._p = C.c_void_p(None)

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def _np_ptr(a: np.ndarray, t):
    return a.ctypes.data_as(t)


def _stream_ptr(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return C.c_void_p(stream.cuda_stream)


# ----------------------------------------------------------------------------- library
def pasta_version() -> str:
    return lib().pasta_version().decode()


_alloc_keepalive = []


def pasta_set_allocator(alloc_fn=None, free_fn=None) -> None:
    """Install python callables ``alloc_fn(nbytes, stream_ptr) -> int`` / ``free_fn(ptr, stream_ptr)``
    as the device allocator hook, or remove the hook when both are None."""
    if alloc_fn is None and free_fn is None:
        check(lib().pasta_set_allocator(None))
        _alloc_keepalive.clear()
        return

    def _a(nbytes, stream, ctx):
        try:
            return alloc_fn(int(nbytes), stream)
        except Exception:
            return None

    def _f(ptr, stream, ctx):
        try:
            free_fn(ptr, stream)
        except Exception:
            pass

    a, f = ALLOC_FN(_a), FREE_FN(_f)
    s = Allocator(a, f, None)
    _alloc_keepalive[:] = [a, f, s]
    check(lib().pasta_set_allocator(C.byref(s)))


def use_torch_allocator() -> None:
    """Route libpasta device allocations through torch's caching allocator."""
    import torch

    def alloc(nbytes, stream):
        return torch.cuda.caching_allocator_alloc(max(nbytes, 1), torch.cuda.current_device(),
                                                  stream or 0)

    def free(ptr, stream):
        torch.cuda.caching_allocator_delete(ptr)

    pasta_set_allocator(alloc, free)


# ----------------------------------------------------------------------------- ingest
def pasta_load_coo(path: str) -> Coo:
    out = C.c_void_p()
    check(lib().pasta_load_coo(path.encode(), C.byref(out)))
    return Coo(out.value)


def pasta_save_coo(x: Coo, path: str) -> None:
    check(lib().pasta_save_coo(x.ptr, path.encode()))


def pasta_coo_from_arrays(dims: Sequence[int], inds: np.ndarray, vals: np.ndarray) -> Coo:
    """Create a device COO tensor from host arrays ``inds`` (u32 [N, M]) and ``vals`` (f32 [M])."""
    dims_a = np.ascontiguousarray(dims, dtype=np.uint32)
    order = dims_a.shape[0]
    vals = np.ascontiguousarray(vals, dtype=np.float32)
    inds = np.ascontiguousarray(inds, dtype=np.uint32).reshape(order, vals.shape[0])
    rows = [np.ascontiguousarray(inds[k]) for k in range(order)]
    arr = (_u32p * max(order, 1))(*[_np_ptr(r, _u32p) for r in rows])
    out = C.c_void_p()
    check(lib().pasta_coo_from_arrays(order, _np_ptr(dims_a, _u32p), vals.shape[0], arr,
                                      _np_ptr(vals, _f32p), C.byref(out)))
    return Coo(out.value)


def pasta_gen_powerlaw(dims: Sequence[int], nnz: int, seed: int, kind: int = 1,
                       initiator: Optional[Sequence[float]] = None, q: float = 0.0,
                       val_lo: float = -1.0, val_hi: float = 1.0, permute: int = 0,
                       alpha: float = 0.0) -> Coo:
    """Synthetic tensor on the GPU: kind 1 Stochastic Kronecker, kind 0 uniform,
    kind 2 slice power law with exponent ``alpha``; see include/pasta.h."""
    dims_a = np.ascontiguousarray(dims, dtype=np.uint32)
    p = GenParams()
    p.kind, p.q, p.permute, p.val_lo, p.val_hi, p.alpha = kind, q, permute, val_lo, val_hi, alpha
    keep = None
    if initiator is not None:
        keep = np.ascontiguousarray(initiator, dtype=np.float64)
        p.initiator = keep.ctypes.data_as(C.POINTER(C.c_double))
    out = C.c_void_p()
    check(lib().pasta_gen_powerlaw(dims_a.shape[0], _np_ptr(dims_a, _u32p), nnz, seed, C.byref(p),
                                   C.byref(out)))
    del keep
    return Coo(out.value)


# ----------------------------------------------------------------------------- formats
def pasta_coo_to_hicoo(x: Coo, block_bits: int = 7) -> Hicoo:
    out = C.c_void_p()
    check(lib().pasta_coo_to_hicoo(x.ptr, block_bits, C.byref(out)))
    return Hicoo(out.value)


def pasta_coo_to_ghicoo(x: Coo, block_bits: int = 7, cmask: int = 0) -> Hicoo:
    """gHiCOO: modes with bit k of ``cmask`` blocked, the rest kept as COO
    coordinates; ``cmask = 0`` lets the library pick (:func:`pasta_ghicoo_auto_mask`)."""
    out = C.c_void_p()
    check(lib().pasta_coo_to_ghicoo(x.ptr, block_bits, cmask, C.byref(out)))
    return Hicoo(out.value)


def pasta_ghicoo_auto_mask(x: Coo, block_bits: int = 7):
    """(cmask, bytes): the storage-minimising gHiCOO mask and its storage in bytes."""
    cm = C.c_uint32()
    nbytes = C.c_uint64()
    check(lib().pasta_ghicoo_auto_mask(x.ptr, block_bits, C.byref(cm), C.byref(nbytes)))
    return cm.value, nbytes.value


def pasta_coo_prepare(x: Coo, mode: int, stream=None) -> None:
    check(lib().pasta_coo_prepare(x.ptr, mode, _stream_ptr(stream)))


def pasta_coo_release_mode(x: Coo, mode: int) -> None:
    """Free the mode-`mode` working copy and its caches (rebuilt on next use)."""
    check(lib().pasta_coo_release_mode(x.ptr, mode))


def pasta_hicoo_prepare(h: Hicoo, mode: int, stream=None) -> None:
    check(lib().pasta_hicoo_prepare(h.ptr, mode, _stream_ptr(stream)))


# ----------------------------------------------------------------------------- MTTKRP
def _factor_ptrs(order, mode, factors, R, dims=None, device=None):
    """Device pointers of the factor list; every non-target factor must be a contiguous
    float32 CUDA tensor [dims[k], R] (all on one device) -- the library reads dims[k] * R
    floats from it (and CP-ALS writes as many), so a short or mistyped factor is rejected here."""
    import torch
    ptrs = (C.c_void_p * order)()
    if len(factors) < order:
        raise PastaError(-1, f"{len(factors)} factors given for an order-{order} tensor")
    for k in range(order):
        f = factors[k] if k < len(factors) else None
        if k == mode:
            ptrs[k] = None
            continue
        if f is None or not isinstance(f, torch.Tensor) or not f.is_cuda:
            raise PastaError(-1, f"factors[{k}] must be a CUDA tensor")
        if f.dtype != torch.float32 or not f.is_contiguous() or f.dim() != 2 or f.shape[1] != R:
            raise PastaError(-1, f"factors[{k}] must be a contiguous float32 [I_k, R] tensor")
        if dims is not None and f.shape[0] != dims[k]:
            raise PastaError(-1, f"factors[{k}] has {f.shape[0]} rows, the tensor's dims[{k}] is {dims[k]}")
        if device is not None and f.device != device:
            raise PastaError(-1, f"factors[{k}] is on {f.device}, expected {device}")
        ptrs[k] = f.data_ptr()
    return ptrs


def _check_out(out, rows, R):
    import torch
    if not (isinstance(out, torch.Tensor) and out.is_cuda and out.dtype == torch.float32
            and out.is_contiguous() and tuple(out.shape) == (rows, R)):
        raise PastaError(-1, f"out must be a contiguous float32 CUDA tensor of shape ({rows}, {R})")


def _rank(factors, mode, R=None):
    if R is not None:
        return int(R)
    for k, f in enumerate(factors):
        if k != mode and f is not None:
            return int(f.shape[1])
    raise PastaError(-1, "no factor matrix given")


def pasta_mttkrp_coo(x: Coo, mode: int, factors, out=None, stream=None, R=None):
    """Mode-`mode` MTTKRP (Eq. 3) on COO; returns ``out`` (float32 [I_mode, R] CUDA tensor)."""
    import torch
    R = _rank(factors, mode, R)
    if not 0 <= mode < x.order:
        raise PastaError(-1, f"mode {mode} >= order {x.order}")
    if out is None:
        dev = next((f.device for k, f in enumerate(factors) if k != mode and f is not None),
                   torch.device("cuda", torch.cuda.current_device()))
        out = torch.empty((x.dims[mode], R), dtype=torch.float32, device=dev)
    _check_out(out, x.dims[mode], R)
    ptrs = _factor_ptrs(x.order, mode, factors, R, x.dims, out.device)
    check(lib().pasta_mttkrp_coo(x.ptr, mode, ptrs, R, C.c_void_p(out.data_ptr()),
                                 _stream_ptr(stream)))
    return out


def pasta_mttkrp_coo_bcast(x: Coo, mode: int, factors, out, dst_ptrs, stream=None, R=None):
    """Fused MTTKRP + all-gather (include/pasta.h): `out` (local CUDA tensor) and every peer
    replica in ``dst_ptrs`` (device addresses from pasta_ipc_open) receive the owned rows."""
    R = _rank(factors, mode, R)
    _check_out(out, x.dims[mode], R)
    ptrs = _factor_ptrs(x.order, mode, factors, R, x.dims, out.device)
    outs = [out.data_ptr()] + [int(p) for p in dst_ptrs]
    op = (C.c_void_p * len(outs))(*outs)
    check(lib().pasta_mttkrp_coo_bcast(x.ptr, mode, ptrs, R, op, len(outs), _stream_ptr(stream)))
    return out


def pasta_mttkrp_hicoo(h: Hicoo, mode: int, factors, out=None, stream=None, R=None):
    """Mode-`mode` MTTKRP on HiCOO (Alg. 3 semantics); returns ``out``."""
    import torch
    R = _rank(factors, mode, R)
    if not 0 <= mode < h.order:
        raise PastaError(-1, f"mode {mode} >= order {h.order}")
    if out is None:
        dev = next((f.device for k, f in enumerate(factors) if k != mode and f is not None),
                   torch.device("cuda", torch.cuda.current_device()))
        out = torch.empty((h.dims[mode], R), dtype=torch.float32, device=dev)
    _check_out(out, h.dims[mode], R)
    ptrs = _factor_ptrs(h.order, mode, factors, R, h.dims, out.device)
    check(lib().pasta_mttkrp_hicoo(h.ptr, mode, ptrs, R, C.c_void_p(out.data_ptr()),
                                   _stream_ptr(stream)))
    return out


def pasta_mttkrp_coo_allmodes_host(x: Coo, host_factors, host_out, stream=None) -> None:
    """All-modes MTTKRP from/to HOST tensors or arrays (float32, contiguous, ideally pinned)."""
    R = int(host_factors[0].shape[1])
    fp = (C.c_void_p * x.order)()
    op = (C.c_void_p * x.order)()
    for k in range(x.order):
        f, o = host_factors[k], host_out[k]
        fp[k] = f.data_ptr() if hasattr(f, "data_ptr") else f.ctypes.data
        op[k] = o.data_ptr() if hasattr(o, "data_ptr") else o.ctypes.data
    check(lib().pasta_mttkrp_coo_allmodes_host(x.ptr, fp, R, op, _stream_ptr(stream)))


def pasta_coo_release_staging(x: Coo) -> None:
    """Free the e2e staging buffers cached in the handle (re-allocated on next use)."""
    check(lib().pasta_coo_release_staging(x.ptr))


def pasta_mttkrp_coo_allmodes_host_batch(x: Coo, steps, stream=None) -> None:
    """`steps` = list of (host_factors, host_out) pairs, each like pasta_mttkrp_coo_allmodes_host's;
    one pipelined call (step i+1's uploads overlap step i's downloads)."""
    n = len(steps)
    if n == 0:
        return
    R = int(steps[0][0][0].shape[1])
    fp = (C.c_void_p * (n * x.order))()
    op = (C.c_void_p * (n * x.order))()
    for i, (hf, ho) in enumerate(steps):
        for k in range(x.order):
            f, o = hf[k], ho[k]
            fp[i * x.order + k] = f.data_ptr() if hasattr(f, "data_ptr") else f.ctypes.data
            op[i * x.order + k] = o.data_ptr() if hasattr(o, "data_ptr") else o.ctypes.data
    check(lib().pasta_mttkrp_coo_allmodes_host_batch(x.ptr, n, fp, R, op, _stream_ptr(stream)))


# ----------------------------------------------------------------------------- multi-GPU
def pasta_coo_row_counts(x: Coo, mode: int) -> np.ndarray:
    counts = np.zeros(x.dims[mode], np.uint64)
    check(lib().pasta_coo_row_counts(x.ptr, mode, _np_ptr(counts, _u64p)))
    return counts


def pasta_row_partition(counts: np.ndarray, nparts: int) -> np.ndarray:
    """Host-only nnz-balanced contiguous row ranges (needs no GPU)."""
    counts = np.ascontiguousarray(counts, dtype=np.uint64)
    bounds = np.zeros(nparts + 1, np.uint32)
    check(lib().pasta_row_partition(counts.shape[0], _np_ptr(counts, _u64p), nparts,
                                    _np_ptr(bounds, _u32p)))
    return bounds


def pasta_coo_partition(x: Coo, mode: int, nparts: int) -> np.ndarray:
    bounds = np.zeros(nparts + 1, np.uint32)
    check(lib().pasta_coo_partition(x.ptr, mode, nparts, _np_ptr(bounds, _u32p)))
    return bounds


def pasta_coo_shard(x: Coo, mode: int, row_lo: int, row_hi: int) -> Coo:
    out = C.c_void_p()
    check(lib().pasta_coo_shard(x.ptr, mode, row_lo, row_hi, C.byref(out)))
    return Coo(out.value)


def pasta_hicoo_shard(h: "Hicoo", mode: int, row_lo: int, row_hi: int) -> "Hicoo":
    """The entries of `h` with row_lo <= i_mode < row_hi as a HiCOO handle (include/pasta.h)."""
    out = C.c_void_p()
    check(lib().pasta_hicoo_shard(h.ptr, mode, row_lo, row_hi, C.byref(out)))
    return Hicoo(out.value)


# ----------------------------------------------------------------------------- introspection
def pasta_coo_info(x: Coo):
    order = C.c_uint32()
    dims = (C.c_uint32 * MAX_ORDER)()
    nnz = C.c_uint64()
    check(lib().pasta_coo_info(x.ptr, C.byref(order), dims, C.byref(nnz)))
    return order.value, tuple(dims[: order.value]), nnz.value


def _export(fn, x, *extra):
    inds = [np.zeros(max(x.nnz, 1), np.uint32) for _ in range(x.order)]
    vals = np.zeros(max(x.nnz, 1), np.float32)
    arr = (_u32p * x.order)(*[_np_ptr(i, _u32p) for i in inds])
    check(fn(x.ptr, *extra, arr, _np_ptr(vals, _f32p)))
    return np.stack([i[: x.nnz] for i in inds]), vals[: x.nnz].copy()


def pasta_coo_export(x: Coo):
    """Canonical arrays -> (inds u32 [N, M], vals f32 [M]) on the host."""
    return _export(lib().pasta_coo_export, x)


def pasta_coo_export_mode(x: Coo, mode: int):
    """Mode-`mode` sorted copy -> (inds, vals) on the host."""
    return _export(lib().pasta_coo_export_mode, x, mode)


def pasta_hicoo_info(h: Hicoo):
    order = C.c_uint32()
    dims = (C.c_uint32 * MAX_ORDER)()
    bb = C.c_uint32()
    nb = C.c_uint64()
    nnz = C.c_uint64()
    check(lib().pasta_hicoo_info(h.ptr, C.byref(order), dims, C.byref(bb), C.byref(nb),
                                 C.byref(nnz)))
    return order.value, tuple(dims[: order.value]), bb.value, nb.value, nnz.value


def pasta_hicoo_export(h: Hicoo) -> dict:
    nb, M, N = h.nblocks, h.nnz, h.order
    bptr = np.zeros(nb + 1, np.uint64)
    binds = [np.zeros(max(nb, 1), np.uint32) for _ in range(N)]
    einds = [np.zeros(max(M, 1), np.uint8) for _ in range(N)]
    vals = np.zeros(max(M, 1), np.float32)
    bp = (_u32p * N)(*[_np_ptr(b, _u32p) for b in binds])
    ep = (_u8p * N)(*[_np_ptr(e, _u8p) for e in einds])
    check(lib().pasta_hicoo_export(h.ptr, _np_ptr(bptr, _u64p), bp, ep, _np_ptr(vals, _f32p)))
    return {"order": N, "block_bits": h.block_bits, "nblocks": nb, "nnz": M, "bptr": bptr,
            "binds": np.stack([b[:nb] for b in binds]), "einds": np.stack([e[:M] for e in einds]),
            "vals": vals[:M].copy()}


def pasta_ghicoo_export(h: Hicoo) -> dict:
    """Canonical gHiCOO arrays (lists indexed by mode; None where a mode has no such array)."""
    nb, M, N, cm = h.nblocks, h.nnz, h.order, h.cmask
    comp = [bool((cm >> k) & 1) for k in range(N)]
    bptr = np.zeros(nb + 1, np.uint64)
    binds = [np.zeros(max(nb, 1), np.uint32) if comp[k] else None for k in range(N)]
    einds = [np.zeros(max(M, 1), np.uint8) if comp[k] else None for k in range(N)]
    uinds = [None if comp[k] else np.zeros(max(M, 1), np.uint32) for k in range(N)]
    bp = (_u32p * N)(*[_np_ptr(b, _u32p) if b is not None else None for b in binds])
    ep = (_u8p * N)(*[_np_ptr(e, _u8p) if e is not None else None for e in einds])
    up = (_u32p * N)(*[_np_ptr(u, _u32p) if u is not None else None for u in uinds])
    vals = np.zeros(max(M, 1), np.float32)
    check(lib().pasta_ghicoo_export(h.ptr, _np_ptr(bptr, _u64p), bp, ep, up, _np_ptr(vals, _f32p)))
    return {"order": N, "block_bits": h.block_bits, "cmask": cm, "nblocks": nb, "nnz": M,
            "bptr": bptr,
            "binds": [b[:nb] if b is not None else None for b in binds],
            "einds": [e[:M] if e is not None else None for e in einds],
            "uinds": [u[:M] if u is not None else None for u in uinds],
            "vals": vals[:M].copy()}


# ----------------------------------------------------------------------------- measurement
def pasta_launch_count() -> int:
    return int(lib().pasta_launch_count())


def pasta_die_map():
    """(die of every SM as an int8 array, SMs per die) of the current device, or (None, (0, 0))
    when no two-die map was measured (the die-split COO MTTKRP is then off)."""
    n = C.c_uint32()
    die = (C.c_int8 * 1024)()
    nd = (C.c_uint32 * 2)()
    check(lib().pasta_die_map(C.byref(n), die, nd))
    if n.value == 0:
        return None, (0, 0)
    return np.array(die[: n.value], np.int8), (nd[0], nd[1])


def pasta_profile_enable(on: bool = True) -> None:
    check(lib().pasta_profile_enable(1 if on else 0))


def pasta_profile_read(which: int, reset: bool = True):
    """Summed device ms and launch count of kernel family `which` (0 COO, 1 HiCOO, 2 zero)."""
    ms = C.c_double()
    n = C.c_uint64()
    check(lib().pasta_profile_read(which, C.byref(ms), C.byref(n), 1 if reset else 0))
    return ms.value, n.value


# ----------------------------------------------------------------------------- CP-ALS
def _dptr(t):
    return C.c_void_p(t.data_ptr())


def pasta_gram(U, G=None, stream=None):
    """G (+)= U^T U in fp64 (R x R CUDA tensor; a fresh zero tensor when G is None)."""
    import torch
    R = int(U.shape[1])
    if G is None:
        G = torch.zeros((R, R), dtype=torch.float64, device=U.device)
    check(lib().pasta_gram(_dptr(U), U.shape[0], R, _dptr(G), _stream_ptr(stream)))
    return G


def pasta_cpals_solve(M, grams, U=None, colsq=None, stream=None):
    """U = M (Hadamard of grams)^-1, colsq += column sums of squares of U."""
    import torch
    rows, R = int(M.shape[0]), int(M.shape[1])
    if U is None:
        U = torch.empty_like(M)
    if colsq is None:
        colsq = torch.zeros(R, dtype=torch.float64, device=M.device)
    gp = (C.c_void_p * max(len(grams), 1))(*[g.data_ptr() for g in grams])
    check(lib().pasta_cpals_solve(_dptr(M), rows, R, gp, len(grams), _dptr(U), _dptr(colsq),
                                  _stream_ptr(stream)))
    return U, colsq


def pasta_cpals_prepare(GM, grams, Wn=None, Gn=None, lam=None, stream=None):
    """Fused CP-ALS algebra (include/pasta.h): from GM = M^T M and the other grams ->
    (Wn fp32 [R, R], Gn fp64 [R, R], lambda fp64 [R]); the factor is then M @ Wn."""
    import torch
    R = int(GM.shape[0])
    dev = GM.device
    if Wn is None:
        Wn = torch.empty((R, R), dtype=torch.float32, device=dev)
    if Gn is None:
        Gn = torch.empty((R, R), dtype=torch.float64, device=dev)
    if lam is None:
        lam = torch.empty(R, dtype=torch.float64, device=dev)
    gp = (C.c_void_p * max(len(grams), 1))(*[g.data_ptr() for g in grams])
    check(lib().pasta_cpals_prepare(_dptr(GM), gp, len(grams), R, _dptr(Wn), _dptr(Gn), _dptr(lam),
                                    _stream_ptr(stream)))
    return Wn, Gn, lam


def pasta_cpals_fit(grams, lam, inner, normx2: float, stream=None) -> float:
    """CP-ALS fit in a libpasta kernel from the (all modes') grams, lambda and <X, Xhat>
    (CUDA fp64 tensors; inner has one element)."""
    gp = (C.c_void_p * len(grams))(*[g.data_ptr() for g in grams])
    fit = C.c_double()
    check(lib().pasta_cpals_fit(gp, len(grams), int(lam.shape[0]), _dptr(lam), _dptr(inner), float(normx2),
                                C.byref(fit), _stream_ptr(stream)))
    return fit.value


def pasta_rows_times(M, Wn, U=None, stream=None):
    """U = M Wn (rows x R times R x R, fp32) in a libpasta kernel."""
    import torch
    if U is None:
        U = torch.empty_like(M)
    check(lib().pasta_rows_times(_dptr(M), int(M.shape[0]), int(M.shape[1]), _dptr(Wn), _dptr(U),
                                 _stream_ptr(stream)))
    return U


def pasta_normalize_columns(U, colsq, lam=None, stream=None):
    import torch
    R = int(U.shape[1])
    if lam is None:
        lam = torch.empty(R, dtype=torch.float64, device=U.device)
    check(lib().pasta_normalize_columns(_dptr(U), U.shape[0], R, _dptr(colsq), _dptr(lam),
                                        _stream_ptr(stream)))
    return lam


def pasta_weighted_inner(A, B, lam, out=None, stream=None):
    import torch
    if out is None:
        out = torch.zeros(1, dtype=torch.float64, device=A.device)
    check(lib().pasta_weighted_inner(_dptr(A), _dptr(B), A.shape[0], int(A.shape[1]), _dptr(lam),
                                     _dptr(out), _stream_ptr(stream)))
    return out


def pasta_coo_norm2(x: Coo) -> float:
    v = C.c_double()
    check(lib().pasta_coo_norm2(x.ptr, C.byref(v)))
    return v.value


def pasta_cpals_coo(x: Coo, factors, max_iters: int = 20, tol: float = 1e-5, stream=None):
    """Single-GPU CP-ALS; `factors` (CUDA float32 [I_k, R], the initial guess) are updated in
    place.  Returns (lambda float64[R], fit per sweep list, sweeps run)."""
    R = int(factors[0].shape[1])
    # CP-ALS overwrites every factor with dims[k] * R floats: validate all of them (mode = -1)
    fp = _factor_ptrs(x.order, -1, factors, R, x.dims, factors[0].device)
    lam = np.zeros(R, np.float64)
    fits = np.zeros(max(max_iters, 1), np.float64)
    it = C.c_uint32()
    check(lib().pasta_cpals_coo(x.ptr, R, max_iters, tol, fp,
                                lam.ctypes.data_as(C.POINTER(C.c_double)),
                                fits.ctypes.data_as(C.POINTER(C.c_double)), C.byref(it),
                                _stream_ptr(stream)))
    return lam, list(fits[: it.value]), it.value


# ----------------------------------------------------------------------------- TTV / TTM
def pasta_coo_fibers(x: Coo, mode: int, stream=None) -> int:
    """Number of mode-`mode` fibers M_F (built once, cached)."""
    nf = C.c_uint64()
    check(lib().pasta_coo_fibers(x.ptr, mode, C.byref(nf), _stream_ptr(stream)))
    return nf.value


def pasta_coo_fiber_export(x: Coo, mode: int) -> np.ndarray:
    """Fiber coordinates u32 [N, M_F] (row `mode` is zero)."""
    nf = pasta_coo_fibers(x, mode)
    arrs = [np.zeros(max(nf, 1), np.uint32) for _ in range(x.order)]
    p = (_u32p * x.order)(*[_np_ptr(a, _u32p) for a in arrs])
    check(lib().pasta_coo_fiber_export(x.ptr, mode, p))
    return np.stack([a[:nf] for a in arrs])


def pasta_ttm_coo(x: Coo, mode: int, U, out=None, stream=None):
    """Semi-sparse TTM (Eq. 2): values [M_F, R] on the mode-`mode` fibers."""
    import torch
    R = int(U.shape[1])
    nf = pasta_coo_fibers(x, mode, stream)
    if out is None:
        out = torch.empty((nf, R), dtype=torch.float32, device=U.device)
    check(lib().pasta_ttm_coo(x.ptr, mode, C.c_void_p(U.data_ptr()), R, C.c_void_p(out.data_ptr()),
                              _stream_ptr(stream)))
    return out


def pasta_ttv_coo(x: Coo, mode: int, v, out=None, stream=None):
    """Semi-sparse TTV (Eq. 1): values [M_F] on the mode-`mode` fibers."""
    import torch
    nf = pasta_coo_fibers(x, mode, stream)
    if out is None:
        out = torch.empty(nf, dtype=torch.float32, device=v.device)
    check(lib().pasta_ttv_coo(x.ptr, mode, C.c_void_p(v.data_ptr()), C.c_void_p(out.data_ptr()),
                              _stream_ptr(stream)))
    return out


# ----------------------------------------------------------------------------- TEW / TS
OPS = {"add": 0, "sub": 1, "mul": 2, "div": 3}


def _op(op):
    return OPS[op] if isinstance(op, str) else int(op)


def _f32_cuda(t, name):
    import torch
    if not (isinstance(t, torch.Tensor) and t.is_cuda and t.dtype == torch.float32 and t.is_contiguous()):
        raise PastaError(-1, f"{name} must be a contiguous float32 CUDA tensor")


def pasta_ts(vals, op, s: float, out=None, stream=None):
    """TS on a value tensor: out = vals op s (IEEE fp32)."""
    import torch
    _f32_cuda(vals, "vals")
    if out is None:
        out = torch.empty_like(vals)
    _f32_cuda(out, "out")
    check(lib().pasta_ts(C.c_void_p(vals.data_ptr()), vals.numel(), _op(op), float(s),
                         C.c_void_p(out.data_ptr()), _stream_ptr(stream)))
    return out


def pasta_tew(a, b, op, out=None, stream=None):
    """Same-pattern TEW on value tensors: out = a op b."""
    import torch
    _f32_cuda(a, "a")
    _f32_cuda(b, "b")
    if a.numel() != b.numel():
        raise PastaError(-1, "a and b differ in length")
    if out is None:
        out = torch.empty_like(a)
    _f32_cuda(out, "out")
    check(lib().pasta_tew(C.c_void_p(a.data_ptr()), C.c_void_p(b.data_ptr()), a.numel(), _op(op),
                          C.c_void_p(out.data_ptr()), _stream_ptr(stream)))
    return out


def pasta_coo_values_ptr(x: Coo) -> int:
    """Device address of x's canonical value array (library-owned)."""
    p = C.c_void_p()
    check(lib().pasta_coo_values(x.ptr, C.byref(p)))
    return p.value or 0


def pasta_coo_ts(x: Coo, op, s: float) -> Coo:
    out = C.c_void_p()
    check(lib().pasta_coo_ts(x.ptr, _op(op), float(s), C.byref(out)))
    return Coo(out.value)


def pasta_coo_tew(x: Coo, y: Coo, op) -> Coo:
    out = C.c_void_p()
    check(lib().pasta_coo_tew(x.ptr, y.ptr, _op(op), C.byref(out)))
    return Coo(out.value)


# ----------------------------------------------------------------------------- peer memory
def pasta_rows_times_bcast(M, row_lo: int, row_hi: int, Wn, dst_ptrs, stream=None) -> None:
    """Rows [row_lo, row_hi) of M @ Wn stored into every replica in ``dst_ptrs`` (device
    addresses: the local factor and peers' factors mapped with :func:`pasta_ipc_open`)."""
    R = int(M.shape[1])
    dp = (C.c_void_p * len(dst_ptrs))(*[int(p) for p in dst_ptrs])
    check(lib().pasta_rows_times_bcast(_dptr(M), int(row_lo), int(row_hi), R, _dptr(Wn), dp,
                                       len(dst_ptrs), _stream_ptr(stream)))


def pasta_bcast_f32(src, dst_ptrs, stream=None) -> None:
    """Copy the contiguous float32 tensor ``src`` to every device address in ``dst_ptrs``
    (peer stores; the P2P all-gather of owned rows)."""
    dp = (C.c_void_p * len(dst_ptrs))(*[int(p) for p in dst_ptrs])
    check(lib().pasta_bcast_f32(_dptr(src), src.numel(), dp, len(dst_ptrs), _stream_ptr(stream)))


class _CudaArray:
    """Zero-copy view of a libpasta device allocation for torch.as_tensor."""

    def __init__(self, ptr: int, shape, typestr="<f4"):
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr,
                                         "data": (int(ptr), False), "version": 3, "strides": None}


def pasta_dev_alloc(shape, dtype="float32"):
    """An IPC-exportable device allocation wrapped as a torch tensor; returns (tensor, ptr).
    Free with :func:`pasta_dev_free` after the last use of the tensor."""
    import torch
    n = int(np.prod(shape))
    p = C.c_void_p()
    check(lib().pasta_dev_alloc(max(n, 1) * 4, C.byref(p)))
    t = torch.as_tensor(_CudaArray(p.value, shape), device="cuda")
    return t, p.value


def pasta_dev_free(ptr: int) -> None:
    check(lib().pasta_dev_free(C.c_void_p(ptr)))


def pasta_ipc_get_handle(ptr: int) -> bytes:
    buf = (C.c_uint8 * 64)()
    check(lib().pasta_ipc_get_handle(C.c_void_p(ptr), buf))
    return bytes(buf)


def pasta_ipc_open(handle: bytes) -> int:
    buf = (C.c_uint8 * 64).from_buffer_copy(handle)
    p = C.c_void_p()
    check(lib().pasta_ipc_open(buf, C.byref(p)))
    return p.value


def pasta_ipc_close(ptr: int) -> None:
    check(lib().pasta_ipc_close(C.c_void_p(ptr)))
