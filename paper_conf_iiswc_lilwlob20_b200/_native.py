"""ctypes declarations for libpasta.so (include/pasta.h).  Loads the in-tree library and
fails loudly if it is missing: there is no CPU or Python fallback for any compute step."""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libpasta.so")

MAX_ORDER = 8

STATUS = {
    0: "PASTA_OK", -1: "PASTA_EINVAL", -2: "PASTA_EIO", -3: "PASTA_EFORMAT", -4: "PASTA_ERANGE",
    -5: "PASTA_ENOMEM", -6: "PASTA_ECUDA", -7: "PASTA_EUNSUPPORTED",
}


class PastaError(RuntimeError):
    """A non-OK pasta_status; ``.code`` is the status, the message is pasta_last_error()."""

    def __init__(self, code: int, msg: str):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code


class GenParams(C.Structure):
    _fields_ = [("kind", C.c_uint32), ("initiator", C.POINTER(C.c_double)), ("q", C.c_double),
                ("permute", C.c_uint32), ("val_lo", C.c_float), ("val_hi", C.c_float),
                ("alpha", C.c_double)]


ALLOC_FN = C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)
FREE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_void_p, C.c_void_p)


class Allocator(C.Structure):
    _fields_ = [("alloc", ALLOC_FN), ("free", FREE_FN), ("ctx", C.c_void_p)]


_u32p = C.POINTER(C.c_uint32)
_u64p = C.POINTER(C.c_uint64)
_f32p = C.POINTER(C.c_float)
_u8p = C.POINTER(C.c_uint8)
_vp = C.c_void_p
_st = C.c_int

# name -> (restype, argtypes); every symbol include/pasta.h declares
SIGNATURES = {
    "pasta_last_error": (C.c_char_p, []),
    "pasta_version": (C.c_char_p, []),
    "pasta_set_allocator": (_st, [C.POINTER(Allocator)]),
    "pasta_load_coo": (_st, [C.c_char_p, C.POINTER(_vp)]),
    "pasta_save_coo": (_st, [_vp, C.c_char_p]),
    "pasta_coo_from_arrays": (_st, [C.c_uint32, _u32p, C.c_uint64, C.POINTER(_u32p), _f32p,
                                    C.POINTER(_vp)]),
    "pasta_gen_powerlaw": (_st, [C.c_uint32, _u32p, C.c_uint64, C.c_uint64, C.POINTER(GenParams),
                                 C.POINTER(_vp)]),
    "pasta_coo_to_hicoo": (_st, [_vp, C.c_uint32, C.POINTER(_vp)]),
    "pasta_coo_to_ghicoo": (_st, [_vp, C.c_uint32, C.c_uint32, C.POINTER(_vp)]),
    "pasta_ghicoo_auto_mask": (_st, [_vp, C.c_uint32, _u32p, _u64p]),
    "pasta_ghicoo_info": (_st, [_vp, _u32p]),
    "pasta_ghicoo_export": (_st, [_vp, _u64p, C.POINTER(_u32p), C.POINTER(_u8p), C.POINTER(_u32p), _f32p]),
    "pasta_coo_prepare": (_st, [_vp, C.c_uint32, _vp]),
    "pasta_hicoo_prepare": (_st, [_vp, C.c_uint32, _vp]),
    "pasta_coo_release_mode": (_st, [_vp, C.c_uint32]),
    "pasta_mttkrp_coo": (_st, [_vp, C.c_uint32, C.POINTER(_vp), C.c_uint32, _vp, _vp]),
    "pasta_mttkrp_hicoo": (_st, [_vp, C.c_uint32, C.POINTER(_vp), C.c_uint32, _vp, _vp]),
    "pasta_mttkrp_coo_bcast": (_st, [_vp, C.c_uint32, C.POINTER(_vp), C.c_uint32, C.POINTER(_vp), C.c_uint32, _vp]),
    "pasta_mttkrp_coo_allmodes_host": (_st, [_vp, C.POINTER(_vp), C.c_uint32, C.POINTER(_vp), _vp]),
    "pasta_mttkrp_coo_allmodes_host_batch": (_st, [_vp, C.c_uint32, C.POINTER(_vp), C.c_uint32,
                                                   C.POINTER(_vp), _vp]),
    "pasta_coo_release_staging": (_st, [_vp]),
    "pasta_coo_row_counts": (_st, [_vp, C.c_uint32, _u64p]),
    "pasta_row_partition": (_st, [C.c_uint32, _u64p, C.c_uint32, _u32p]),
    "pasta_coo_partition": (_st, [_vp, C.c_uint32, C.c_uint32, _u32p]),
    "pasta_coo_shard": (_st, [_vp, C.c_uint32, C.c_uint32, C.c_uint32, C.POINTER(_vp)]),
    "pasta_hicoo_shard": (_st, [_vp, C.c_uint32, C.c_uint32, C.c_uint32, C.POINTER(_vp)]),
    "pasta_ts": (_st, [_vp, C.c_uint64, C.c_uint32, C.c_float, _vp, _vp]),
    "pasta_tew": (_st, [_vp, _vp, C.c_uint64, C.c_uint32, _vp, _vp]),
    "pasta_coo_values": (_st, [_vp, C.POINTER(_vp)]),
    "pasta_coo_ts": (_st, [_vp, C.c_uint32, C.c_float, C.POINTER(_vp)]),
    "pasta_coo_tew": (_st, [_vp, _vp, C.c_uint32, C.POINTER(_vp)]),
    "pasta_coo_info": (_st, [_vp, _u32p, _u32p, _u64p]),
    "pasta_coo_export": (_st, [_vp, C.POINTER(_u32p), _f32p]),
    "pasta_coo_export_mode": (_st, [_vp, C.c_uint32, C.POINTER(_u32p), _f32p]),
    "pasta_hicoo_info": (_st, [_vp, _u32p, _u32p, _u32p, _u64p, _u64p]),
    "pasta_hicoo_export": (_st, [_vp, _u64p, C.POINTER(_u32p), C.POINTER(_u8p), _f32p]),
    "pasta_coo_free": (None, [_vp]),
    "pasta_hicoo_free": (None, [_vp]),
    "pasta_gram": (_st, [_vp, C.c_uint64, C.c_uint32, _vp, _vp]),
    "pasta_cpals_solve": (_st, [_vp, C.c_uint64, C.c_uint32, C.POINTER(_vp), C.c_uint32, _vp, _vp, _vp]),
    "pasta_cpals_prepare": (_st, [_vp, C.POINTER(_vp), C.c_uint32, C.c_uint32, _vp, _vp, _vp, _vp]),
    "pasta_rows_times": (_st, [_vp, C.c_uint64, C.c_uint32, _vp, _vp, _vp]),
    "pasta_cpals_fit": (_st, [C.POINTER(_vp), C.c_uint32, C.c_uint32, _vp, _vp, C.c_double,
                              C.POINTER(C.c_double), _vp]),
    "pasta_rows_times_bcast": (_st, [_vp, C.c_uint64, C.c_uint64, C.c_uint32, _vp, C.POINTER(_vp),
                                     C.c_uint32, _vp]),
    "pasta_bcast_f32": (_st, [_vp, C.c_uint64, C.POINTER(_vp), C.c_uint32, _vp]),
    "pasta_dev_alloc": (_st, [C.c_uint64, C.POINTER(_vp)]),
    "pasta_dev_free": (_st, [_vp]),
    "pasta_ipc_get_handle": (_st, [_vp, _vp]),
    "pasta_ipc_open": (_st, [_vp, C.POINTER(_vp)]),
    "pasta_ipc_close": (_st, [_vp]),
    "pasta_normalize_columns": (_st, [_vp, C.c_uint64, C.c_uint32, _vp, _vp, _vp]),
    "pasta_weighted_inner": (_st, [_vp, _vp, C.c_uint64, C.c_uint32, _vp, _vp, _vp]),
    "pasta_coo_norm2": (_st, [_vp, C.POINTER(C.c_double)]),
    "pasta_cpals_coo": (_st, [_vp, C.c_uint32, C.c_uint32, C.c_double, C.POINTER(_vp),
                              C.POINTER(C.c_double), C.POINTER(C.c_double), _u32p, _vp]),
    "pasta_coo_fibers": (_st, [_vp, C.c_uint32, _u64p, _vp]),
    "pasta_coo_fiber_export": (_st, [_vp, C.c_uint32, C.POINTER(_u32p)]),
    "pasta_ttm_coo": (_st, [_vp, C.c_uint32, _vp, C.c_uint32, _vp, _vp]),
    "pasta_ttv_coo": (_st, [_vp, C.c_uint32, _vp, _vp, _vp]),
    "pasta_launch_count": (C.c_uint64, []),
    "pasta_die_map": (_st, [_u32p, C.POINTER(C.c_int8), _u32p]),
    "pasta_profile_enable": (_st, [C.c_int]),
    "pasta_profile_read": (_st, [C.c_uint32, C.POINTER(C.c_double), _u64p, C.c_int]),
}

_lib = None


def lib() -> C.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(
                f"libpasta.so not found at {LIB_PATH}: build it with `make` or "
                "`python -c 'import __graft_entry__ as g; g.build()'` (no CPU fallback exists)")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def check(status: int) -> None:
    if status != 0:
        msg = lib().pasta_last_error()
        raise PastaError(status, msg.decode() if msg else "")
