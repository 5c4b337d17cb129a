"""CPU oracle for the Eirene batched B+tree path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
`--impl reference` legs may import this package.  The product path
(paper_conf_ppopp_zhangz0lzl23_b200) never imports it and shares no code with
it: the oracle is plain C++ (oracle/eirene_oracle.cpp) behind ctypes.

Engines (see eirene_oracle.h for the paper citations):
  MapOracle      -- the plain definition, std::map
  BTreeOracle    -- textbook sequential B+tree (split / borrow / merge); timed baseline
  combine_apply  -- Algorithm 1 step by step on a MapOracle,
                    exposing the issued set per segment
Parity status is recorded in DESIGN.md §3.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "eirene_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
NOT_FOUND = np.uint64(0xFFFFFFFFFFFFFFFF)

_u64p = ctypes.POINTER(ctypes.c_uint64)
_u32p = ctypes.POINTER(ctypes.c_uint32)
_u8p = ctypes.POINTER(ctypes.c_uint8)
_vp = ctypes.c_void_p


def build(force: bool = False) -> str:
    """Compile the oracle with g++ (-O2, plain sequential C++17)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "eirene_oracle.h"))):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        sig = {
            "orc_map_new": (_vp, []), "orc_map_free": (None, [_vp]),
            "orc_map_load": (ctypes.c_int, [_vp, _u64p, _u64p, ctypes.c_uint64]),
            "orc_map_apply": (ctypes.c_int, [_vp, _u8p, _u64p, _u64p, ctypes.c_uint64, _u64p]),
            "orc_map_size": (ctypes.c_uint64, [_vp]),
            "orc_map_scan": (ctypes.c_uint64, [_vp, ctypes.c_uint64, ctypes.c_uint64, _u64p, _u64p, ctypes.c_uint64]),
            "orc_bt_new": (_vp, [ctypes.c_int]), "orc_bt_free": (None, [_vp]),
            "orc_bt_load": (ctypes.c_int, [_vp, _u64p, _u64p, ctypes.c_uint64]),
            "orc_bt_apply": (ctypes.c_int, [_vp, _u8p, _u64p, _u64p, ctypes.c_uint64, _u64p]),
            "orc_bt_size": (ctypes.c_uint64, [_vp]),
            "orc_bt_scan": (ctypes.c_uint64, [_vp, ctypes.c_uint64, ctypes.c_uint64, _u64p, _u64p, ctypes.c_uint64]),
            "orc_bt_check": (ctypes.c_int, [_vp]),
            "orc_bt_height": (ctypes.c_int, [_vp]),
            "orc_bt_corrupt": (ctypes.c_int, [_vp, ctypes.c_int]),
            "orc_comb_apply": (ctypes.c_int, [_vp, _u8p, _u64p, _u64p, ctypes.c_uint64, _u64p, _u32p, _u32p,
                                              _u64p, _u8p, _u64p, _u64p, _u64p]),
            "orc_map_apply_range": (ctypes.c_int, [_vp, _u8p, _u64p, _u64p, ctypes.c_uint64, _u64p, ctypes.c_uint32,
                                                   _u64p, _u64p]),
            "orc_bt_apply_range": (ctypes.c_int, [_vp, _u8p, _u64p, _u64p, ctypes.c_uint64, _u64p, ctypes.c_uint32,
                                                  _u64p, _u64p]),
            "orc_comb_apply_range": (ctypes.c_int, [_vp, _u8p, _u64p, _u64p, ctypes.c_uint64, _u64p, ctypes.c_uint32,
                                                    _u64p, _u64p, _u64p]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _p(a: np.ndarray | None, t):
    if a is None:
        return ctypes.cast(None, t)
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(t)


def _req(ops, keys, vals):
    ops = np.ascontiguousarray(ops, dtype=np.uint8)
    keys = np.ascontiguousarray(keys, dtype=np.uint64)
    vals = np.ascontiguousarray(vals, dtype=np.uint64)
    assert ops.shape == keys.shape == vals.shape
    return ops, keys, vals


class _Engine:
    _pre = ""

    def __init__(self, h):
        self.h = h
        self.L = lib()

    def __del__(self):
        if getattr(self, "h", None):
            getattr(self.L, f"orc_{self._pre}_free")(self.h)
            self.h = None

    def load(self, keys, vals):
        keys = np.ascontiguousarray(keys, dtype=np.uint64)
        vals = np.ascontiguousarray(vals, dtype=np.uint64)
        rc = getattr(self.L, f"orc_{self._pre}_load")(self.h, _p(keys, _u64p), _p(vals, _u64p), keys.size)
        if rc != 0:
            raise ValueError("oracle load: keys must be strictly increasing and != UINT64_MAX")

    def apply(self, ops, keys, vals) -> np.ndarray:
        ops, keys, vals = _req(ops, keys, vals)
        res = np.empty(ops.size, dtype=np.uint64)
        rc = getattr(self.L, f"orc_{self._pre}_apply")(self.h, _p(ops, _u8p), _p(keys, _u64p),
                                                       _p(vals, _u64p), ops.size, _p(res, _u64p))
        if rc != 0:
            raise ValueError("oracle apply: invalid request (op > 3, key == UINT64_MAX, or upsert of UINT64_MAX)")
        return res

    def apply_range(self, ops, keys, vals, cap: int):
        """Batch with range queries (op RANGE = 4: key = l, val = u, inclusive).
        Returns (results[n], rkeys[n, cap], rvals[n, cap]); for a range request
        results[i] = pairs written (first `cap` of [l, u] in key order), rows of
        non-range requests and unused slots are left zero."""
        ops, keys, vals = _req(ops, keys, vals)
        n = ops.size
        res = np.empty(n, dtype=np.uint64)
        rk = np.zeros((n, max(cap, 1)), dtype=np.uint64)
        rv = np.zeros((n, max(cap, 1)), dtype=np.uint64)
        rc = getattr(self.L, f"orc_{self._pre}_apply_range")(self.h, _p(ops, _u8p), _p(keys, _u64p), _p(vals, _u64p),
                                                             n, _p(res, _u64p), cap, _p(rk, _u64p), _p(rv, _u64p))
        if rc != 0:
            raise ValueError("oracle apply_range: invalid request")
        return res, rk[:, :cap], rv[:, :cap]

    def size(self) -> int:
        return int(getattr(self.L, f"orc_{self._pre}_size")(self.h))

    def scan(self, lo: int = 0, hi: int = 0xFFFFFFFFFFFFFFFE):
        f = getattr(self.L, f"orc_{self._pre}_scan")
        cnt = int(f(self.h, lo, hi, _p(None, _u64p), _p(None, _u64p), 0))
        k = np.empty(cnt, dtype=np.uint64)
        v = np.empty(cnt, dtype=np.uint64)
        f(self.h, lo, hi, _p(k, _u64p), _p(v, _u64p), cnt)
        return k, v


class MapOracle(_Engine):
    """Engine (i): the plain sequential definition on a std::map."""
    _pre = "map"

    def __init__(self):
        super().__init__(lib().orc_map_new())


class BTreeOracle(_Engine):
    """Engine (ii): textbook sequential B+tree with fanout F."""
    _pre = "bt"

    def __init__(self, fanout: int = 16):
        h = lib().orc_bt_new(fanout)
        if not h:
            raise ValueError("fanout must be in [3, 64]")
        super().__init__(h)

    def check(self) -> int:
        return int(self.L.orc_bt_check(self.h))

    def height(self) -> int:
        return int(self.L.orc_bt_height(self.h))

    def corrupt(self, kind: int) -> int:
        return int(self.L.orc_bt_corrupt(self.h, kind))


def combine_apply(m: MapOracle, ops, keys, vals):
    """Engine (iii): Algorithm 1 on MapOracle `m` (mutated).  Returns a dict with
    results[n] (ts order), sorted_ts[n], seg[n] (segment of each sorted position),
    issued_key/op/val[m] per segment, n_issued, n_issued_w."""
    ops, keys, vals = _req(ops, keys, vals)
    n = ops.size
    res = np.empty(n, dtype=np.uint64)
    sts = np.empty(n, dtype=np.uint32)
    seg = np.empty(n, dtype=np.uint32)
    ik = np.empty(n, dtype=np.uint64)
    io = np.empty(n, dtype=np.uint8)
    iv = np.empty(n, dtype=np.uint64)
    ni = ctypes.c_uint64(0)
    nw = ctypes.c_uint64(0)
    rc = lib().orc_comb_apply(m.h, _p(ops, _u8p), _p(keys, _u64p), _p(vals, _u64p), n, _p(res, _u64p),
                              _p(sts, _u32p), _p(seg, _u32p), _p(ik, _u64p), _p(io, _u8p), _p(iv, _u64p),
                              ctypes.byref(ni), ctypes.byref(nw))
    if rc != 0:
        raise ValueError("oracle combine: invalid request")
    mi = ni.value
    return dict(results=res, sorted_ts=sts, seg=seg, issued_key=ik[:mi], issued_op=io[:mi],
                issued_val=iv[:mi], n_issued=mi, n_issued_w=nw.value)


RANGE = 4


def combine_apply_range(m: MapOracle, ops, keys, vals, cap: int):
    """Engine (iii) with range queries: the artificial-query mechanism of
    P:920-938 around Algorithm 1, on MapOracle `m` (mutated).  Returns
    (results[n], rkeys[n, cap], rvals[n, cap], n_artificial)."""
    ops, keys, vals = _req(ops, keys, vals)
    n = ops.size
    res = np.empty(n, dtype=np.uint64)
    rk = np.zeros((n, max(cap, 1)), dtype=np.uint64)
    rv = np.zeros((n, max(cap, 1)), dtype=np.uint64)
    na = ctypes.c_uint64(0)
    rc = lib().orc_comb_apply_range(m.h, _p(ops, _u8p), _p(keys, _u64p), _p(vals, _u64p), n, _p(res, _u64p), cap,
                                    _p(rk, _u64p), _p(rv, _u64p), ctypes.byref(na))
    if rc != 0:
        raise ValueError("oracle combine_apply_range: invalid request")
    return res, rk[:, :cap], rv[:, :cap], na.value
