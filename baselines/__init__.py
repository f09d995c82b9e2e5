"""CPU baselines that are NOT the oracle: the paper's own OpenMP COO-MTTKRP,
fp32 with `omp atomic`, on all host cores -- reported by bench.py as `cpu_omp`, clearly apart
from `cpu_baseline` (the fp64 oracle).  No product code imports this package."""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "omp_mttkrp.c")
_SO = os.path.join(_HERE, "libomp_mttkrp.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O3", "-march=native", "-fopenmp", "-fPIC", "-shared", "-o", _SO, _SRC])
    return _SO


def _L():
    global _lib
    if _lib is None:
        lib = C.CDLL(build())
        u32p, f32p = C.POINTER(C.c_uint32), C.POINTER(C.c_float)
        lib.omp_mttkrp_coo.restype = C.c_int
        lib.omp_mttkrp_coo.argtypes = [C.c_uint32, u32p, C.c_uint64, C.POINTER(u32p), f32p, C.c_uint32,
                                       C.POINTER(f32p), C.c_uint32, f32p]
        lib.omp_threads.restype = C.c_int
        _lib = lib
    return _lib


def threads() -> int:
    return int(_L().omp_threads())


def mttkrp(dims, inds, vals, mode, factors):
    """fp32 COO-MTTKRP-OMP; returns out float32 [dims[mode], R]."""
    dims = np.ascontiguousarray(dims, dtype=np.uint32)
    inds = np.ascontiguousarray(inds, dtype=np.uint32)
    vals = np.ascontiguousarray(vals, dtype=np.float32)
    R = int(next(f for k, f in enumerate(factors) if k != mode).shape[1])
    fl = [np.ascontiguousarray(factors[k] if k != mode else np.zeros((1, R), np.float32), dtype=np.float32)
          for k in range(len(dims))]
    out = np.empty((int(dims[mode]), R), np.float32)
    u32p, f32p = C.POINTER(C.c_uint32), C.POINTER(C.c_float)
    rows = [inds[k] for k in range(inds.shape[0])]
    ip = (u32p * len(rows))(*[r.ctypes.data_as(u32p) for r in rows])
    fp = (f32p * len(fl))(*[f.ctypes.data_as(f32p) for f in fl])
    rc = _L().omp_mttkrp_coo(len(dims), dims.ctypes.data_as(u32p), vals.shape[0], ip, vals.ctypes.data_as(f32p),
                             mode, fp, R, out.ctypes.data_as(f32p))
    if rc != 0:
        raise ValueError("omp_mttkrp_coo failed")
    return out
