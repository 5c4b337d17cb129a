"""ctypes binding of include/eirene.h (argument marshalling only).

Every function of the C ABI is exposed under the same name.  The library is
the in-tree libeirene.so built by `build.py`; importing this module never
falls back to anything else: if the library is missing or cannot be loaded,
`lib()` raises.
"""
from __future__ import annotations

import ctypes
import os
import re

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
# EIRENE_LIB: an alternative build of the same library (A/B experiments); default: the in-tree one
LIB_PATH = os.environ.get("EIRENE_LIB") or os.path.join(PKG, "libeirene.so")
# the 32-bit key / value build (-DEIRENE_KEY32): same API, eirene_key_t = uint32_t
LIB32_PATH = os.environ.get("EIRENE_LIB32") or os.path.join(PKG, "libeirene32.so")
HEADER = os.path.join(ROOT, "include", "eirene.h")

EIRENE_OK, EIRENE_EINVAL, EIRENE_ENOMEM, EIRENE_EFULL, EIRENE_ESTATE, EIRENE_ECUDA, EIRENE_EINTERNAL = (
    0, -1, -2, -3, -4, -5, -6)
EIRENE_QUERY, EIRENE_UPDATE, EIRENE_INSERT, EIRENE_DELETE, EIRENE_RANGE = 0, 1, 2, 3, 4
EIRENE_F_REGROUP, EIRENE_F_STATS, EIRENE_F_FORCE_STM, EIRENE_F_TIMING, EIRENE_F_ITERWARP = 1, 2, 4, 8, 16
EIRENE_F_PIPELINE = 32
NOT_FOUND = 0xFFFFFFFFFFFFFFFF

_u64 = ctypes.c_uint64
_u32 = ctypes.c_uint32
_vp = ctypes.c_void_p
_int = ctypes.c_int


class eirene_config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("fanout", _u32), ("max_keys", _u64), ("max_batch", _u32),
                ("retry_threshold", _u32), ("flags", _u32), ("key_lo", _u64), ("key_hi", _u64),
                ("iter_rgs", _u32)]


class eirene_batch_stats(ctypes.Structure):
    _fields_ = [("status", ctypes.c_int32), ("n", _u32), ("distinct", _u64), ("issued_q", _u64),
                ("issued_w", _u64), ("leaf_runs", _u64), ("retries", _u64), ("stm_fallbacks", _u64),
                ("leaf_splits", _u64), ("inner_splits", _u64), ("new_leaves", _u64), ("new_inner", _u64),
                ("height", _u32), ("launches", _u32), ("stage_ms", ctypes.c_float * 8),
                ("ranges", _u64), ("artificial", _u64), ("trav_steps", _u64), ("rg_vertical", _u64),
                ("rg_horizontal", _u64), ("device_ns", _u64), ("t_begin_ns", _u64), ("t_end_ns", _u64), ("nins", _u64), ("ndelp", _u64)]

    def to_dict(self) -> dict:
        d = {f: getattr(self, f) for f, _ in self._fields_ if f != "stage_ms"}
        d["stage_ms"] = list(self.stage_ms)
        return d


class eirene_tree_info(ctypes.Structure):
    _fields_ = [("height", _u32), ("root", _u32), ("leaves", _u64), ("inner", _u64), ("leaf_cap", _u64),
                ("inner_cap", _u64), ("launches", _u64), ("device_bytes", _u64)]


EIRENE_IPC_HANDLE_BYTES = 64   # include/eirene.h

_SIGS = {
    "eirene_default_config": (None, [ctypes.POINTER(eirene_config)]),
    "eirene_create": (_int, [ctypes.POINTER(eirene_config), ctypes.POINTER(_vp)]),
    "eirene_bulk_load": (_int, [_vp, _vp, _vp, _u64, ctypes.c_float, _vp]),
    "eirene_submit_batch": (_int, [_vp, _vp, _vp, _vp, _u32, _vp, _vp, ctypes.POINTER(_u64)]),
    "eirene_submit_batch_host": (_int, [_vp, _vp, _vp, _vp, _u32, _vp, _vp, ctypes.POINTER(_u64)]),
    "eirene_prepare_batch": (_int, [_vp, _u32, _int]),
    "eirene_submit_batch_range": (_int, [_vp, _vp, _vp, _vp, _u32, _vp, _u32, _vp, _vp, _vp, ctypes.POINTER(_u64)]),
    "eirene_results": (_int, [_vp, _u64, ctypes.POINTER(eirene_batch_stats)]),
    "eirene_scan": (_int, [_vp, _u64, _u64, _vp, _vp, _u64, ctypes.POINTER(_u64), _vp]),
    "eirene_check_invariants": (_int, [_vp, ctypes.POINTER(_u64)]),
    "eirene_get_info": (_int, [_vp, ctypes.POINTER(eirene_tree_info)]),
    "eirene_set_flags": (_int, [_vp, _u32]),
    "eirene_probe_gather": (_int, [_vp, _u64, _u32, ctypes.c_int, _u64, _vp]),
    "eirene_destroy": (_int, [_vp]),
    "eirene_strerror": (ctypes.c_char_p, [_int]),
    "eirene_last_cuda_error": (ctypes.c_char_p, []),
    "eirene_route_partition": (_int, [_vp, _vp, _vp, _vp, _u32, _vp, _int, _vp, _vp, _vp, _vp, _vp, _vp, _vp]),
    "eirene_route_unpermute": (_int, [_vp, _vp, _vp, _u32, _vp, _vp]),
    "eirene_route_partition_packed": (_int, [_vp, _vp, _vp, _vp, _u32, _vp, _int, _vp, _vp, _vp, _vp]),
    "eirene_route_unpack": (_int, [_vp, _vp, _u32, _vp, _vp, _vp, _vp]),
    "eirene_batch_status_async": (_int, [_vp, _u64, _vp, _vp]),
    "eirene_debug_phases": (_int, [_vp, _vp, _u32]),
    "eirene_stream_wait_batch": (_int, [_vp, _u64, _vp]),
    "eirene_route_arena_create": (_int, [_vp, _int, _int, _u32, ctypes.POINTER(_vp), _vp]),
    "eirene_route_arena_open_ipc": (_int, [_vp, _vp, ctypes.POINTER(_vp)]),
    "eirene_route_arena_connect": (_int, [_vp, _vp]),
    "eirene_route_push": (_int, [_vp, _vp, _vp, _vp, _u32, _vp, _vp, _vp]),
    "eirene_route_pull": (_int, [_vp, _vp, _vp, _vp, _u32, ctypes.POINTER(_u32), ctypes.POINTER(_u32), _vp]),
    "eirene_route_push_results": (_int, [_vp, _vp, _vp]),
    "eirene_route_unpermute_arena": (_int, [_vp, _vp, _u32, _vp, _vp]),
}

_libs: dict = {}


def header_functions() -> list[str]:
    """Names of the functions include/eirene.h declares."""
    with open(HEADER) as f:
        text = f.read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(eirene_[a-z_]+)\s*\(", text)))


def lib(key_bits: int = 64) -> ctypes.CDLL:
    """Load libeirene.so (key_bits 64) or libeirene32.so (32); raises if it was not built."""
    if key_bits not in _libs:
        path = {64: LIB_PATH, 32: LIB32_PATH}[key_bits]
        if not os.path.exists(path):
            raise RuntimeError(f"{path} is missing: run `python -m paper_conf_ppopp_zhangz0lzl23_b200.build` "
                               "(there is no CPU fallback)")
        L = ctypes.CDLL(path)
        for name, (res, args) in _SIGS.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _libs[key_bits] = L
    return _libs[key_bits]


class EireneError(RuntimeError):
    def __init__(self, code: int, where: str):
        L = lib()
        msg = L.eirene_strerror(code).decode()
        if code == EIRENE_ECUDA:
            msg += ": " + L.eirene_last_cuda_error().decode()
        super().__init__(f"{where}: {msg} ({code})")
        self.code = code


def check(code: int, where: str) -> int:
    if code != EIRENE_OK:
        raise EireneError(code, where)
    return code
