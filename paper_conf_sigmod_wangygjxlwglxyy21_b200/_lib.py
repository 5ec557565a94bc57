"""ctypes loader for libmv.so (the C ABI of include/mv.h).  Argument marshalling only.

The product path has no fallback: if libmv.so is missing or cannot be loaded this raises.
"""
from __future__ import annotations

import ctypes as C
import os
import re

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libmv.so")
HEADER = os.path.join(os.path.dirname(_PKG), "include", "mv.h")

MV_L2, MV_IP = 0, 1
MV_IVF_FLAT, MV_IVF_SQ8, MV_IVF_PQ = 0, 1, 2
STATUS = {0: "MV_OK", -1: "MV_EINVAL", -2: "MV_ESTATE", -3: "MV_ENOMEM", -4: "MV_ECUDA", -5: "MV_ENCCL"}


class MvError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


_lib = None

_P = C.c_void_p

ALLOC_FN = C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)
FREE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_void_p, C.c_void_p)


class MvAllocator(C.Structure):
    """mv_allocator of include/mv.h."""
    _fields_ = [("alloc", ALLOC_FN), ("free", FREE_FN), ("ctx", C.c_void_p)]

_SIGS = {
    "mv_index_create": (C.c_int, [C.c_int32, C.c_int, C.c_int, C.c_int32, C.c_int32, C.POINTER(MvAllocator),
                                  C.POINTER(C.c_void_p)]),
    "mv_index_set_option": (C.c_int, [_P, C.c_char_p, C.c_int64]),
    "mv_index_set_centroids": (C.c_int, [_P, _P]),
    "mv_index_train_sq8": (C.c_int, [_P, _P, C.c_int64]),
    "mv_index_set_sq8": (C.c_int, [_P, _P, _P]),
    "mv_index_get_sq8": (C.c_int, [_P, _P, _P]),
    "mv_index_add": (C.c_int, [_P, _P, _P, C.c_int64, _P]),
    "mv_search": (C.c_int, [_P, _P, C.c_int64, C.c_int32, C.c_int32, _P, C.c_int64, _P, _P, _P]),
    "mv_search_probes": (C.c_int, [_P, _P, C.c_int64, C.c_int32, _P, _P]),
    "mv_search_with_probes": (C.c_int, [_P, _P, C.c_int64, C.c_int32, C.c_int32, _P, _P, C.c_int64, _P, _P, _P]),
    "mv_merge_topk": (C.c_int, [C.c_int, _P, _P, C.c_int32, C.c_int64, C.c_int32, _P, _P, _P]),
    "mv_index_set_pq": (C.c_int, [_P, C.c_int32, _P]),
    "mv_index_get_pq": (C.c_int, [_P, _P, _P]),
    "mv_index_train_pq": (C.c_int, [_P, C.c_int32, _P, C.c_int64, C.c_int32]),
    "mv_kmeans": (C.c_int, [_P, C.c_int64, C.c_int32, C.c_int, C.c_int32, C.c_int32, C.c_int32, _P, C.c_int32, _P]),
    "mv_attr_bitset": (C.c_int, [_P, _P, C.c_int64, C.c_int64, C.c_int64, _P, C.c_int64, _P]),
    "mv_fuse_rows": (C.c_int, [C.POINTER(C.c_void_p), C.POINTER(C.c_int32), C.POINTER(C.c_float), C.c_int32,
                               C.c_int64, _P, _P]),
    "mv_index_ntotal": (C.c_int64, [_P]),
    "mv_index_storage": (C.c_int, [_P, _P, _P, _P]),
    "mv_index_destroy": (None, [_P]),
    "mv_profile_enable": (C.c_int, [_P, C.c_int]),
    "mv_index_describe": (C.c_int, [_P, C.c_char_p, C.c_size_t]),
    "mv_profile_read": (C.c_int, [_P, _P, _P, _P, C.c_int]),
    "mv_profile_counters": (C.c_int, [_P, _P, C.c_int]),
    "mv_last_error": (C.c_char_p, []),
    "mv_version": (C.c_char_p, []),
}


def header_symbols() -> list[str]:
    """Every entry point include/mv.h declares (MV_API ... mv_xxx( )."""
    with open(HEADER) as f:
        txt = f.read()
    return sorted(set(re.findall(r"^MV_API[^(]*?\b(mv_\w+)\s*\(", txt, flags=re.M)))


def load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_sigmod_wangygjxlwglxyy21_b200.build`"
                          " (there is no CPU fallback)")
    lib = C.CDLL(LIB_PATH)
    for name, (res, args) in _SIGS.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    _lib = lib
    return lib


def check(status: int):
    if status != 0:
        raise MvError(status, (load().mv_last_error() or b"").decode())
