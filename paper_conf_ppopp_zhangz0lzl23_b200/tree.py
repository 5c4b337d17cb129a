"""Python face of the C ABI: an Eirene tree on one GPU, fed with torch tensors.

PyTorch only provides device memory and streams here; every step of the batch
pipeline runs in the sm_100a kernels behind libeirene.so (include/eirene.h).

    t = EireneTree(max_keys=1 << 24, max_batch=1 << 20)
    t.bulk_load(keys_u64, vals_u64)                   # torch.uint64 on cuda
    ticket = t.submit(ops_u8, keys_u64, vals_u64, results_u64)
    stats = t.results(ticket)                         # waits, returns a dict
    k, v = t.scan()                                   # in-order contents
"""
from __future__ import annotations

import ctypes

import torch

from . import _ffi
from ._ffi import check

U64_MAX = (1 << 64) - 1


def _ptr(t: torch.Tensor | None) -> int | None:
    return None if t is None else t.data_ptr()


def _need(t: torch.Tensor, dtype: torch.dtype, dev: torch.device, name: str, n: int | None = None):
    if t.dtype != dtype:
        raise TypeError(f"{name}: expected {dtype}, got {t.dtype}")
    if t.device != dev:
        raise ValueError(f"{name}: expected device {dev}, got {t.device}")
    if not t.is_contiguous():
        raise ValueError(f"{name}: must be contiguous")
    if n is not None and t.numel() < n:
        raise ValueError(f"{name}: needs {n} elements")


class EireneTree:
    """One B+tree (or one key-range shard of it) resident on one GPU."""

    def __init__(self, max_keys: int = 1 << 24, max_batch: int = 1 << 20, device: int | None = None,
                 retry_threshold: int = 4, regroup: bool = True, stats: bool = True, force_stm: bool = False,
                 timing: bool = False, key_lo: int = 0, key_hi: int = U64_MAX, iterwarp: bool = False,
                 iter_rgs: int = 0, pipeline: bool = False, key_bits: int = 64):
        # key_bits 32: libeirene32.so (32-bit keys and values); tensors torch.uint32
        L = _ffi.lib(key_bits)
        self.key_bits = key_bits
        self.kdtype = torch.uint32 if key_bits == 32 else torch.uint64
        self.not_found = (1 << key_bits) - 1
        if device is None:
            device = torch.cuda.current_device()
        self.device = torch.device("cuda", device)
        cfg = _ffi.eirene_config()
        L.eirene_default_config(ctypes.byref(cfg))
        cfg.device = device
        cfg.max_keys = max_keys
        cfg.max_batch = max_batch
        cfg.retry_threshold = retry_threshold
        cfg.flags = ((_ffi.EIRENE_F_REGROUP if regroup else 0) | (_ffi.EIRENE_F_STATS if stats else 0) |
                     (_ffi.EIRENE_F_FORCE_STM if force_stm else 0) | (_ffi.EIRENE_F_TIMING if timing else 0) |
                     (_ffi.EIRENE_F_ITERWARP if iterwarp else 0) | (_ffi.EIRENE_F_PIPELINE if pipeline else 0))
        cfg.iter_rgs = iter_rgs
        cfg.key_lo = key_lo
        cfg.key_hi = key_hi
        self.cfg = cfg
        h = ctypes.c_void_p()
        check(L.eirene_create(ctypes.byref(cfg), ctypes.byref(h)), "eirene_create")
        self._h = h
        self._L = L
        self.max_batch = max_batch

    # ---------------------------------------------------------------- lifecycle
    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            self._L.eirene_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def _stream(self, stream):
        s = stream if stream is not None else torch.cuda.current_stream(self.device)
        return s.cuda_stream

    # ---------------------------------------------------------------- ABI calls
    def bulk_load(self, keys: torch.Tensor, vals: torch.Tensor, leaf_fill: float = 1.0, stream=None):
        _need(keys, self.kdtype, self.device, "keys")
        _need(vals, self.kdtype, self.device, "vals", keys.numel())
        check(self._L.eirene_bulk_load(self._h, _ptr(keys), _ptr(vals), keys.numel(), leaf_fill,
                                       self._stream(stream)), "eirene_bulk_load")

    def submit(self, ops: torch.Tensor, keys: torch.Tensor, vals: torch.Tensor, results: torch.Tensor,
               stream=None) -> int:
        n = ops.numel()
        _need(ops, torch.uint8, self.device, "ops")
        _need(keys, self.kdtype, self.device, "keys", n)
        _need(vals, self.kdtype, self.device, "vals", n)
        _need(results, self.kdtype, self.device, "results", n)
        tk = ctypes.c_uint64()
        check(self._L.eirene_submit_batch(self._h, _ptr(ops), _ptr(keys), _ptr(vals), n, _ptr(results),
                                          self._stream(stream), ctypes.byref(tk)), "eirene_submit_batch")
        return tk.value

    def prepare(self, n: int, ranges: bool = False):
        """Capture the batch graph for n-request batches ahead of the first one (no launch)."""
        check(self._L.eirene_prepare_batch(self._h, n, 1 if ranges else 0), "eirene_prepare_batch")

    def submit_range(self, ops: torch.Tensor, keys: torch.Tensor, vals: torch.Tensor, results: torch.Tensor,
                     cap: int, range_keys: torch.Tensor, range_vals: torch.Tensor, stream=None) -> int:
        """Batch that may hold range queries (op RANGE = 4, key = l, val = u, inclusive):
        range_keys / range_vals are [n, cap] u64; row i receives the first results[i] pairs of R(l, u)."""
        n = ops.numel()
        _need(ops, torch.uint8, self.device, "ops")
        _need(keys, self.kdtype, self.device, "keys", n)
        _need(vals, self.kdtype, self.device, "vals", n)
        _need(results, self.kdtype, self.device, "results", n)
        _need(range_keys, self.kdtype, self.device, "range_keys", n * cap)
        _need(range_vals, self.kdtype, self.device, "range_vals", n * cap)
        tk = ctypes.c_uint64()
        check(self._L.eirene_submit_batch_range(self._h, _ptr(ops), _ptr(keys), _ptr(vals), n, _ptr(results), cap,
                                                _ptr(range_keys), _ptr(range_vals), self._stream(stream),
                                                ctypes.byref(tk)), "eirene_submit_batch_range")
        return tk.value

    def apply_range(self, ops, keys, vals, cap: int, stream=None):
        """submit_range + results: returns (results, range_keys [n, cap], range_vals [n, cap], stats)."""
        n = ops.numel()
        res = torch.empty(n, dtype=self.kdtype, device=self.device)
        rk = torch.zeros((n, cap), dtype=self.kdtype, device=self.device)
        rv = torch.zeros((n, cap), dtype=self.kdtype, device=self.device)
        tk = self.submit_range(ops, keys, vals, res, cap, rk, rv, stream)
        return res, rk, rv, self.results(tk)

    def submit_host(self, ops: torch.Tensor, keys: torch.Tensor, vals: torch.Tensor, results: torch.Tensor,
                    stream=None) -> int:
        """Host (ideally pinned) buffers: the library copies them in on its own copy stream, runs the
        batch on `stream` and copies the results out on its own d2h stream; results are valid after
        results(ticket).  Pinned values are read zero-copy (only upserts' values are ever read)."""
        n = ops.numel()
        cpu = torch.device("cpu")
        _need(ops, torch.uint8, cpu, "ops")
        _need(keys, self.kdtype, cpu, "keys", n)
        _need(vals, self.kdtype, cpu, "vals", n)
        _need(results, self.kdtype, cpu, "results", n)
        tk = ctypes.c_uint64()
        check(self._L.eirene_submit_batch_host(self._h, _ptr(ops), _ptr(keys), _ptr(vals), n, _ptr(results),
                                               self._stream(stream), ctypes.byref(tk)), "eirene_submit_batch_host")
        return tk.value

    def stream_wait(self, ticket: int, stream=None):
        """Order `stream` (default: current) after batch `ticket` on the device (needed with pipeline=True
        before consuming its results there)."""
        check(self._L.eirene_stream_wait_batch(self._h, ticket, self._stream(stream)), "eirene_stream_wait_batch")

    def results(self, ticket: int, raise_on_error: bool = True) -> dict:
        st = _ffi.eirene_batch_stats()
        rc = self._L.eirene_results(self._h, ticket, ctypes.byref(st))
        if rc != _ffi.EIRENE_OK and raise_on_error:
            raise _ffi.EireneError(rc, "eirene_results")
        d = st.to_dict()
        d["rc"] = rc
        return d

    def apply(self, ops, keys, vals, results=None, stream=None):
        """submit + results: returns (results tensor, stats dict)."""
        if results is None:
            results = torch.empty(ops.numel(), dtype=self.kdtype, device=self.device)
        tk = self.submit(ops, keys, vals, results, stream)
        return results, self.results(tk)

    def scan(self, lo: int = 0, hi: int = U64_MAX - 1, stream=None):
        hi = min(hi, self.not_found - 1)
        cnt = ctypes.c_uint64()
        s = self._stream(stream)
        check(self._L.eirene_scan(self._h, lo, hi, None, None, 0, ctypes.byref(cnt), s), "eirene_scan")
        n = cnt.value
        k = torch.empty(max(n, 1), dtype=self.kdtype, device=self.device)
        v = torch.empty(max(n, 1), dtype=self.kdtype, device=self.device)
        check(self._L.eirene_scan(self._h, lo, hi, _ptr(k), _ptr(v), n, ctypes.byref(cnt), s), "eirene_scan")
        return k[:n], v[:n]

    def check_invariants(self) -> tuple[int, int]:
        nk = ctypes.c_uint64()
        rc = self._L.eirene_check_invariants(self._h, ctypes.byref(nk))
        if rc < 0:
            raise _ffi.EireneError(rc, "eirene_check_invariants")
        return rc, nk.value

    def set_flags(self, regroup: bool | None = None, stats: bool | None = None, force_stm: bool | None = None,
                  timing: bool | None = None, iterwarp: bool | None = None):
        f = self.cfg.flags
        for on, bit in ((regroup, _ffi.EIRENE_F_REGROUP), (stats, _ffi.EIRENE_F_STATS),
                        (force_stm, _ffi.EIRENE_F_FORCE_STM), (timing, _ffi.EIRENE_F_TIMING),
                        (iterwarp, _ffi.EIRENE_F_ITERWARP)):   # (pipelining is fixed at create)
            if on is not None:
                f = (f | bit) if on else (f & ~bit)
        self.cfg.flags = f
        check(self._L.eirene_set_flags(self._h, f), "eirene_set_flags")

    def info(self) -> dict:
        i = _ffi.eirene_tree_info()
        check(self._L.eirene_get_info(self._h, ctypes.byref(i)), "eirene_get_info")
        return {f: getattr(i, f) for f, _ in i._fields_}

    # ---------------------------------------------------------------- routing
    def route_partition(self, ops, keys, vals, splitters: torch.Tensor | None, P: int, stream=None,
                        invalid: torch.Tensor | None = None):
        """Stable partition by destination shard; returns (send_ops, send_keys, send_vals, perm, counts).
        `invalid` (int32[1] on the device) is set to 1 if any request is invalid."""
        n = ops.numel()
        dev = self.device
        sops = torch.empty(n, dtype=torch.uint8, device=dev)
        skeys = torch.empty(n, dtype=torch.uint64, device=dev)
        svals = torch.empty(n, dtype=torch.uint64, device=dev)
        perm = torch.empty(n, dtype=torch.int32, device=dev)
        counts = torch.empty(P, dtype=torch.int32, device=dev)
        check(self._L.eirene_route_partition(self._h, _ptr(ops), _ptr(keys), _ptr(vals), n,
                                             _ptr(splitters) if splitters is not None else None, P, _ptr(sops),
                                             _ptr(skeys), _ptr(svals), _ptr(perm), _ptr(counts), _ptr(invalid),
                                             self._stream(stream)), "eirene_route_partition")
        return sops, skeys, svals, perm, counts

    def route_unpermute(self, recv: torch.Tensor, perm: torch.Tensor, out: torch.Tensor | None = None, stream=None):
        n = recv.numel()
        if out is None:
            out = torch.empty(n, dtype=torch.uint64, device=self.device)
        check(self._L.eirene_route_unpermute(self._h, _ptr(recv), _ptr(perm), n, _ptr(out), self._stream(stream)),
              "eirene_route_unpermute")
        return out

    def route_partition_packed(self, ops, keys, vals, splitters: torch.Tensor | None, P: int, stream=None):
        """Partition for ONE payload exchange: returns (send_rec u64[3n] of {key, value, op} records grouped by
        destination, perm int32[n], counts2 int32[2P] = (count, validity flag) per destination)."""
        n = ops.numel()
        dev = self.device
        rec = torch.empty(3 * n, dtype=torch.uint64, device=dev)
        perm = torch.empty(n, dtype=torch.int32, device=dev)
        counts2 = torch.empty(2 * P, dtype=torch.int32, device=dev)
        check(self._L.eirene_route_partition_packed(self._h, _ptr(ops), _ptr(keys), _ptr(vals), n,
                                                    _ptr(splitters) if splitters is not None else None, P,
                                                    _ptr(rec), _ptr(perm), _ptr(counts2), self._stream(stream)),
              "eirene_route_partition_packed")
        return rec, perm, counts2

    def route_unpack(self, rec: torch.Tensor, n: int, stream=None):
        """Split n received {key, value, op} records into (ops u8, keys u64, vals u64)."""
        dev = self.device
        ops = torch.empty(n, dtype=torch.uint8, device=dev)
        keys = torch.empty(n, dtype=torch.uint64, device=dev)
        vals = torch.empty(n, dtype=torch.uint64, device=dev)
        check(self._L.eirene_route_unpack(self._h, _ptr(rec), n, _ptr(ops), _ptr(keys), _ptr(vals),
                                          self._stream(stream)), "eirene_route_unpack")
        return ops, keys, vals

    # ------------------------------------------- fused routing over peer memory (NEXT(3))
    def route_arena_create(self, P: int, rank: int, cap: int) -> tuple[int, bytes]:
        """This rank's receive arena: (device address, CUDA IPC handle bytes)."""
        addr = ctypes.c_void_p()
        ipc = ctypes.create_string_buffer(_ffi.EIRENE_IPC_HANDLE_BYTES)
        check(self._L.eirene_route_arena_create(self._h, P, rank, cap, ctypes.byref(addr), ipc),
              "eirene_route_arena_create")
        return int(addr.value), bytes(ipc.raw)

    def route_arena_open_ipc(self, handle: bytes) -> int:
        addr = ctypes.c_void_p()
        buf = ctypes.create_string_buffer(bytes(handle), _ffi.EIRENE_IPC_HANDLE_BYTES)
        check(self._L.eirene_route_arena_open_ipc(self._h, buf, ctypes.byref(addr)), "eirene_route_arena_open_ipc")
        return int(addr.value)

    def route_arena_connect(self, peer_addrs: list[int]):
        arr = (ctypes.c_void_p * len(peer_addrs))(*peer_addrs)
        check(self._L.eirene_route_arena_connect(self._h, arr), "eirene_route_arena_connect")

    def route_push(self, ops, keys, vals, splitters: torch.Tensor | None, perm: torch.Tensor, stream=None):
        """Partition this slice and store every request into its destination's arena; perm int32[n] out."""
        n = ops.numel()
        check(self._L.eirene_route_push(self._h, _ptr(ops), _ptr(keys), _ptr(vals), n,
                                        _ptr(splitters) if splitters is not None else None, _ptr(perm),
                                        self._stream(stream)), "eirene_route_push")

    def route_pull(self, ops, keys, vals, stream=None) -> tuple[int, int]:
        """Compact the records pushed to this rank into ops/keys/vals (capacity = their length);
        returns (n, invalid).  One host synchronisation."""
        n = _ffi._u32()
        inv = _ffi._u32()
        check(self._L.eirene_route_pull(self._h, _ptr(ops), _ptr(keys), _ptr(vals), ops.numel(), ctypes.byref(n),
                                        ctypes.byref(inv), self._stream(stream)), "eirene_route_pull")
        return int(n.value), int(inv.value)

    def route_push_results(self, results: torch.Tensor | None, stream=None):
        check(self._L.eirene_route_push_results(self._h, _ptr(results) if results is not None else None,
                                                self._stream(stream)), "eirene_route_push_results")

    def route_unpermute_arena(self, perm: torch.Tensor, out: torch.Tensor, stream=None):
        check(self._L.eirene_route_unpermute_arena(self._h, _ptr(perm), perm.numel(), _ptr(out),
                                                   self._stream(stream)), "eirene_route_unpermute_arena")
        return out

    def status_async(self, ticket: int, out: torch.Tensor, stream=None):
        """Enqueue a copy of batch `ticket`'s final status into out (int32[1] on the device), no host sync."""
        check(self._L.eirene_batch_status_async(self._h, ticket, _ptr(out), self._stream(stream)),
              "eirene_batch_status_async")
        return out
