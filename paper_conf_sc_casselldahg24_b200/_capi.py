"""ctypes binding of include/nbody.h -- argument marshalling only.

Every function here has the C name and forwards to libnbody_b200.so; there
is no Python or CPU implementation of any stage behind it.  If the shared
library is missing or cannot load, every call raises (no fallback).
"""
from __future__ import annotations

import ctypes as C
import os

from . import build as _build

NBODY_OK = 0
NBODY_EINVAL = -1
NBODY_ENOMEM = -2
NBODY_ECUDA = -3
NBODY_ENCCL = -4
NBODY_ESTATE = -5

NBODY_OPT_KEY_BITS = 1
NBODY_OPT_STREAM = 2
NBODY_OPT_USE_GRAPH = 3
NBODY_OPT_TRAVERSAL = 4
NBODY_OPT_TIMING = 5
NBODY_OPT_BUILD = 6
NBODY_OPT_SORT_EVERY = 7
NBODY_OPT_MULTIPOLE = 8
NBODY_OPT_BALANCE = 9
NBODY_OPT_PRECISION = 10

NBODY_WS_QUAD = 1
NBODY_WS_XFER = 2
NBODY_WS_FP64 = 4

_STATUS = {0: "NBODY_OK", -1: "NBODY_EINVAL", -2: "NBODY_ENOMEM", -3: "NBODY_ECUDA", -4: "NBODY_ENCCL",
           -5: "NBODY_ESTATE"}


class NBodyError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


class nbody_stats(C.Structure):
    _fields_ = [("n", C.c_int64), ("key_bits", C.c_int), ("levels", C.c_int), ("steps", C.c_int64),
                ("interactions", C.c_uint64), ("ms_bbox_keys", C.c_float), ("ms_sort", C.c_float),
                ("ms_build", C.c_float), ("ms_force", C.c_float), ("ms_update", C.c_float),
                ("kernels_per_step", C.c_int), ("lane_util", C.c_float)]


_P = C.c_void_p
_I64 = C.c_int64
_S = C.c_int

# name -> (restype, argtypes)
SIGNATURES = {
    "nbody_version": (C.c_int, []),
    "nbody_select_device": (_S, [C.c_int]),
    "nbody_debug_force_stats": (C.c_int, [_P, C.c_int]),
    "nbody_create": (_S, [_I64, C.c_double, C.c_double, C.c_double, C.POINTER(_P)]),
    "nbody_create_ws": (_S, [_I64, C.c_double, C.c_double, C.c_double, _P, C.c_size_t, C.POINTER(_P)]),
    "nbody_workspace_bytes": (C.c_size_t, [_I64, C.c_int, C.c_int]),
    "nbody_workspace_bytes_ex": (C.c_size_t, [_I64, C.c_int, C.c_int, C.c_uint]),
    "nbody_attach_comm": (_S, [_P, _P, C.c_int, C.c_int]),
    "nbody_allpairs_accel": (_S, [_P, _P, _I64, _P, _P]),
    "nbody_set_option": (_S, [_P, C.c_int, _I64]),
    "nbody_set_bodies": (_S, [_P, _P, _P, _P]),
    "nbody_set_bodies_async": (_S, [_P, _P, _P, _P]),
    "nbody_get_positions_async": (_S, [_P, _P]),
    "nbody_compute_accel": (_S, [_P]),
    "nbody_step": (_S, [_P, C.c_int]),
    "nbody_sync": (_S, [_P]),
    "nbody_get_accel": (_S, [_P, _P]),
    "nbody_get_positions": (_S, [_P, _P]),
    "nbody_get_velocities": (_S, [_P, _P]),
    "nbody_get_interactions": (_S, [_P, _P]),
    "nbody_get_state": (_S, [_P, _P, _P]),
    "nbody_set_bodies64": (_S, [_P, _P, _P, _P]),
    "nbody_get_accel64": (_S, [_P, _P]),
    "nbody_get_positions64": (_S, [_P, _P]),
    "nbody_get_velocities64": (_S, [_P, _P]),
    "nbody_get_state64": (_S, [_P, _P, _P]),
    "nbody_set_state": (_S, [_P, _P, _P, _I64]),
    "nbody_set_state64": (_S, [_P, _P, _P, _I64]),
    "nbody_debug_level64": (_S, [_P, C.c_int, C.POINTER(_I64), _P, _P]),
    "nbody_get_stats": (_S, [_P, C.POINTER(nbody_stats)]),
    "nbody_direct_accel": (_S, [_P, _P, _I64, _P]),
    "nbody_partition": (_S, [_I64, C.c_int, C.c_int, C.POINTER(_I64), C.POINTER(_I64)]),
    "nbody_has_nccl": (C.c_int, []),
    "nbody_nccl_unique_id": (_S, [_P]),
    "nbody_attach_nccl": (_S, [_P, _P, C.c_int, C.c_int]),
    "nbody_set_partition": (_S, [_P, C.c_int, C.c_int]),
    "nbody_get_partition": (_S, [_P, C.POINTER(C.c_int), C.POINTER(C.c_int), C.POINTER(_I64),
                                 C.POINTER(_I64)]),
    "nbody_copy_owned": (_S, [_P, _P]),
    "nbody_peer_handle": (_S, [_P, _P]),
    "nbody_attach_peers": (_S, [_P, _P, C.c_int, C.c_int]),
    "nbody_attach_peers_local": (_S, [C.POINTER(_P), C.c_int]),
    "nbody_exchange_mode": (C.c_int, [_P]),
    "nbody_debug_quad": (_S, [_P, C.c_int, _P]),
    "nbody_debug_keys": (_S, [_P, _P]),
    "nbody_debug_perm": (_S, [_P, _P]),
    "nbody_debug_level": (_S, [_P, C.c_int, C.POINTER(_I64), _P, _P, _P]),
    "nbody_last_error": (C.c_char_p, [_P]),
    "nbody_destroy": (None, [_P]),
}

_lib = None


def load(build_if_needed: bool = True):
    """Load libnbody_b200.so (building it in-tree with nvcc if stale)."""
    global _lib
    if _lib is None:
        path = _build.LIB
        if build_if_needed and _build.stale():
            _build.build()
        if not os.path.exists(path):
            raise ImportError(f"{path} is missing: run `python -m paper_conf_sc_casselldahg24_b200.build`")
        lib = C.CDLL(path)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(lib, name)
            f.restype = res
            f.argtypes = args
        _lib = lib
    return _lib


def check(ctx, status: int):
    if status != NBODY_OK:
        msg = load().nbody_last_error(ctx).decode() if ctx else ""
        raise NBodyError(status, msg)


def __getattr__(name):  # module-level passthrough: _capi.nbody_step(...)
    if name in SIGNATURES:
        return getattr(load(), name)
    raise AttributeError(name)
