"""ctypes binding of include/mm.h -- argument marshalling only.

Every step of the matching path runs in lib/libmm.so (CUDA, sm_100a).  There
is no CPU fallback: if the library is missing or cannot be loaded, importing
the engine raises.
"""
from __future__ import annotations

import ctypes
import os

from . import _build

MM_SEM_MPI = 0
MM_SEM_NOWILD_ORDERED = 1
MM_SEM_NOWILD_UNORDERED = 2

MM_OK = 0
MM_ERR_ARG = 1
MM_ERR_CUDA = 2
MM_ERR_CAPACITY = 3
MM_ERR_NOMEM = 4
MM_ERR_STATE = 5

MM_OPT_MPI_KERNEL = 1
MM_OPT_FLAT_KERNEL = 2
MM_OPT_PIPELINE_CHUNKS = 3
MM_OPT_HOST_OUT = 4
MM_HOST_OUT_STAGED, MM_HOST_OUT_MAPPED = 0, 1
MM_FLAT_KERNEL_BUCKETED, MM_FLAT_KERNEL_GLOBAL = 0, 1
MM_MPI_KERNEL_AUTO, MM_MPI_KERNEL_MATRIX, MM_MPI_KERNEL_FIFO = 0, 1, 2

MM_NO_MATCH = -1
MM_ANY_SOURCE = 0xFFFFFFFF
MM_ANY_TAG = 0xFFFF
MM_MPI_MAX_MSGS = 24576

(MM_Q_N_OUT, MM_Q_N_MATCHED, MM_Q_RESID_RECV, MM_Q_RESID_MSG, MM_Q_ERROR, MM_Q_KERNEL_NS, MM_Q_KERNEL_RUNS,
 MM_Q_LAUNCHES, MM_Q_FALLBACKS, MM_Q_COUNT) = range(10)

# name -> (restype, argtypes); must list every function include/mm.h declares
_P = ctypes.c_void_p
_I32 = ctypes.c_int32
_I64 = ctypes.c_int64
SIGNATURES = {
    "mm_create": (ctypes.c_int, [ctypes.POINTER(_P), _I32, _I32, _I64, _I64, _P]),
    "mm_post_recvs": (ctypes.c_int, [_P, _P, _P, _P, _I64]),
    "mm_push_msgs": (ctypes.c_int, [_P, _P, _P, _P, _I64]),
    "mm_match_batch": (ctypes.c_int, [_P, _P, _P, _I64, _P]),
    "mm_reset": (ctypes.c_int, [_P]),
    "mm_query": (ctypes.c_int, [_P, _P]),
    "mm_destroy": (ctypes.c_int, [_P]),
    "mm_route": (ctypes.c_int, [_P, _P, _I64, _I32, _I32, _I64, _P, _P, _P, _P]),
    "mm_set_option": (ctypes.c_int, [_P, _I32, _I64]),
    "mm_strerror": (ctypes.c_char_p, [ctypes.c_int]),
    "mm_version": (ctypes.c_char_p, []),
}

_lib = None


class MMError(RuntimeError):
    def __init__(self, code, where):
        self.code = code
        super().__init__("%s failed: %s (code %d)" % (where, strerror(code), code))


def lib_path():
    return _build.LIB


def load(build_if_missing=True):
    """Load lib/libmm.so (building it with nvcc if it is missing or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("MM_LIB", _build.LIB)  # MM_LIB: profiling builds only
    if build_if_missing and path == _build.LIB and _build.stale():
        _build.build_library()
    if not os.path.exists(path):
        raise RuntimeError("libmm.so not found at %s: the CUDA extension is required "
                           "(no CPU fallback exists)" % path)
    L = ctypes.CDLL(path)
    for name, (res, args) in SIGNATURES.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def strerror(code):
    return load().mm_strerror(code).decode()


def check(code, where):
    if code != MM_OK:
        raise MMError(code, where)
    return code
