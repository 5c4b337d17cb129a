"""Key-range sharded Eirene over torch.distributed (one process per GPU).

SURVEY.md §8(e): requests on different keys are independent (§8(c)), so the
tree is partitioned by key range -- shard r owns [splitter[r-1], splitter[r]),
the splitters being equal-count quantiles of the bulk-loaded keys -- and each
batch needs one exchange step each way:

  1. every rank holds the contiguous timestamp slice r of the global batch;
  2. route_partition_packed (CUDA kernels) stably groups the slice by
     destination shard (dest = upper_bound(splitters, key)) into 24 B
     {key, value, op} records and counts per destination;
  3. ONE all_to_all_single of (count, validity flag) per destination: the
     receive counts, and every rank's flag (a bad request anywhere rejects the
     global batch everywhere, before any shard applies) -- the one host sync;
  4. ONE all_to_all_single of the records (NCCL over NVLink 5 / NVSwitch),
     route_unpack on the receiver;
     the receiver's concatenation in source-rank order is timestamp-ordered,
     so the shard's stable (key, ts) sort keeps linearizability (per-key
     locality of linearizability, Herlihy & Wing [17]);
  5. the shard runs the single-GPU hot path (eirene_submit_batch); its final
     status is copied on the device and all-reduced (MIN), so an EFULL /
     EINTERNAL on one shard fails the global batch on every rank and no rank
     raises alone while the others wait in a collective;
  6. all_to_all_single returns the results; route_unpermute (CUDA kernel)
     puts them back in the slice's timestamp order.

With fused=True (bench.py's default at N > 1) steps 2-4 and 6 run over peer
memory instead: every rank's receive arena is mapped
into every other rank by CUDA IPC (NVLink 5 / NVSwitch), the partition kernel
stores each request straight into its destination's arena
(eirene_route_push), the shard pulls its records after a one-word barrier
(eirene_route_pull: the one host sync) and pushes the results straight back
(eirene_route_push_results); the status all-reduce is the second barrier.
No payload collective runs at all.

The engine (per-shard tree) and router are injectable so the host-side logic
(splitters, count exchange, concatenation order, inverse permutation) can be
tested on CPU with the gloo backend; the product path uses EireneTree and its
CUDA routing kernels and never falls back to anything else.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

U64_MAX = (1 << 64) - 1


def splitters_for(keys: np.ndarray, world: int) -> np.ndarray:
    """P-1 equal-count quantiles of the sorted bulk-loaded keys (u64)."""
    n = keys.size
    return np.array([keys[(r + 1) * n // world] for r in range(world - 1)], dtype=np.uint64)


def shard_range(splitters: np.ndarray, rank: int, world: int) -> tuple[int, int]:
    lo = 0 if rank == 0 else int(splitters[rank - 1])
    hi = U64_MAX if rank == world - 1 else int(splitters[rank])
    return lo, hi


def _i64(t: torch.Tensor) -> torch.Tensor:
    return t.view(torch.int64)


class ShardedEirene:
    """One key-range shard of a distributed Eirene tree on this rank's device.

    keys/vals: the GLOBAL sorted bulk-load arrays (numpy u64, identical on every
    rank); this rank loads its own range.  max_batch: requests per rank per
    batch (the shard accepts up to world * max_batch routed requests).
    """

    def __init__(self, keys: np.ndarray, vals: np.ndarray, max_batch: int, device=None, group=None,
                 engine=None, router=None, fused: bool = False, **tree_kw):
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.device = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.splitters_np = splitters_for(keys, self.world)
        self.lo, self.hi = shard_range(self.splitters_np, self.rank, self.world)
        sel = (keys >= np.uint64(self.lo)) & ((keys < np.uint64(self.hi)) if self.hi != U64_MAX else True)
        my_k, my_v = np.ascontiguousarray(keys[sel]), np.ascontiguousarray(vals[sel])
        self.max_batch = max_batch
        if engine is None:
            from .tree import EireneTree
            engine = EireneTree(max_keys=max(2 * my_k.size, 1 << 16), max_batch=self.world * max_batch,
                                device=self.device.index, key_lo=self.lo, key_hi=self.hi, **tree_kw)
        self.engine = engine
        self.router = router if router is not None else engine
        if my_k.size:
            self.engine.bulk_load(torch.from_numpy(my_k).to(self.device), torch.from_numpy(my_v).to(self.device))
        self.splitters = torch.from_numpy(self.splitters_np if self.world > 1 else np.zeros(1, np.uint64)).to(self.device)
        self.fused = fused
        if fused:
            # every rank must map every peer's arena; if any rank cannot (no CUDA IPC between the processes,
            # no peer access), ALL ranks take the NCCL exchange instead -- decided together
            ok = 1
            try:
                self._connect_arenas()
            except Exception as e:   # noqa: BLE001 -- reported, and agreed on below
                ok = 0
                self.route_error = f"{type(e).__name__}: {e}"
            if self.world > 1:
                flag = torch.tensor([ok], dtype=torch.int32,
                                    device=self.device if self.device.type == "cuda" else "cpu")
                dist.all_reduce(flag, op=dist.ReduceOp.MIN, group=self.group)
                ok = int(flag.item())
            if not ok:
                self.fused = False

    def _connect_arenas(self):
        """Fused routing: every rank's receive arena, mapped into every other rank's
        process over CUDA IPC (peer memory over NVLink 5 / NVSwitch), so the partition kernel pushes the
        requests straight into their shards and the shards push the results straight back."""
        addr, ipc = self.engine.route_arena_create(self.world, self.rank, self.max_batch)
        handles = [ipc]
        if self.world > 1:
            handles = [None] * self.world
            dist.all_gather_object(handles, ipc, group=self.group)   # (collective: before anything can fail)
        addrs = [addr if r == self.rank else self.engine.route_arena_open_ipc(handles[r]) for r in range(self.world)]
        self.engine.route_arena_connect(addrs)
        self._tok = torch.zeros(1, dtype=torch.int32, device=self.device)

    def _barrier(self):
        """Stream-ordered barrier: no rank passes it before every rank's preceding kernels (its pushes into
        the peers' arenas) are complete."""
        if self.world > 1:
            dist.all_reduce(self._tok, group=self.group)

    def _submit_fused(self, ops, keys, vals, results) -> "ShardedTicket":
        """One global batch with the fused push: partition + peer stores (no payload collective), barrier,
        pull (the one host sync), the shard's batch, results pushed back, barrier (the status all-reduce),
        unpermute from the arena."""
        P, n, dev = self.world, int(ops.numel()), self.device
        perm = torch.empty(n, dtype=torch.int32, device=dev)
        self.engine.route_push(ops, keys, vals, self.splitters, perm)
        self._barrier()
        cap = P * self.max_batch
        rops = torch.empty(cap, dtype=torch.uint8, device=dev)
        rkeys = torch.empty(cap, dtype=torch.uint64, device=dev)
        rvals = torch.empty(cap, dtype=torch.uint64, device=dev)
        nrecv, invalid = self.engine.route_pull(rops, rkeys, rvals)
        if invalid:   # every rank saw every source's flag: all reject the global batch
            # (a barrier still: no source may push the next batch into an arena before its owner has read
            # this batch's slots)
            self._barrier()
            return ShardedTicket(self, None, None, n, rejected=-1)
        rres = torch.empty(max(nrecv, 1), dtype=torch.uint64, device=dev)
        status = torch.zeros(1, dtype=torch.int32, device=dev)
        tk = None
        if nrecv:
            tk = self.engine.submit(rops[:nrecv], rkeys[:nrecv], rvals[:nrecv], rres[:nrecv])
            self.engine.status_async(tk, status)   # (orders the current stream after the batch)
        self.engine.route_push_results(rres)
        if P > 1:   # the status all-reduce doubles as the barrier after the result pushes
            dist.all_reduce(status, op=dist.ReduceOp.MIN, group=self.group)
        self.engine.route_unpermute_arena(perm, results)
        return ShardedTicket(self, tk, status, n, keep=(perm, rops, rkeys, rvals, rres))

    def submit(self, ops: torch.Tensor, keys: torch.Tensor, vals: torch.Tensor, results: torch.Tensor) -> "ShardedTicket":
        """Process this rank's timestamp slice of a global batch; `results` (slice order) is valid once the
        returned ticket's results() returns.  Collective: every rank calls it for every global batch in the
        same order.  ONE host synchronisation per batch (the receive counts the payload exchange needs);
        everything else is stream-ordered on the current stream:

          route_partition_packed -> all_to_all(counts + validity flags) -> [host: counts]
          -> all_to_all(24 B records) -> route_unpack -> submit (shard's hot path)
          -> status copy + all_reduce(MIN) -> all_to_all(results) -> route_unpermute
        """
        if self.fused:
            return self._submit_fused(ops, keys, vals, results)
        P = self.world
        n = int(ops.numel())
        rec, perm, cnt2 = self.router.route_partition_packed(ops, keys, vals, self.splitters, P)
        recv2 = torch.empty_like(cnt2)
        if P > 1:
            dist.all_to_all_single(recv2, cnt2, group=self.group)
        else:
            recv2.copy_(cnt2)
        both = torch.cat([cnt2, recv2]).cpu().numpy().astype(np.int64)   # the one host sync
        sc = both[0:2 * P:2].tolist()
        rcv = both[2 * P::2].tolist()
        invalid = int(both[2 * P + 1::2].max())   # every rank's flag: all ranks agree
        if invalid:
            return ShardedTicket(self, None, None, n, rejected=-1)
        nrecv = int(sum(rcv))
        dev = self.device
        rrec = torch.empty(3 * nrecv, dtype=torch.uint64, device=dev)
        if P > 1:
            dist.all_to_all_single(_i64(rrec), _i64(rec), [3 * c for c in rcv], [3 * c for c in sc],
                                   group=self.group)
        else:
            rrec.copy_(rec)
        rops, rkeys, rvals = self.router.route_unpack(rrec, nrecv)
        rres = torch.empty(nrecv, dtype=torch.uint64, device=dev)
        status = torch.zeros(1, dtype=torch.int32, device=dev)
        tk = None
        if nrecv:
            tk = self.engine.submit(rops, rkeys, rvals, rres)
            self.engine.status_async(tk, status)   # (orders the current stream after the batch)
        if P > 1:
            # EFULL / EINTERNAL / CUDA failure on one shard fails the global batch on every rank
            # (statuses are <= 0: the minimum is the error, if any) -- no rank raises alone
            dist.all_reduce(status, op=dist.ReduceOp.MIN, group=self.group)
        back = torch.empty(n, dtype=torch.uint64, device=dev)
        if P > 1:
            dist.all_to_all_single(_i64(back), _i64(rres), sc, rcv, group=self.group)
        else:
            back.copy_(rres)
        self.router.route_unpermute(back, perm, out=results)
        # the ticket keeps every buffer of the batch alive until its results are read
        return ShardedTicket(self, tk, status, n, keep=(rec, perm, rrec, rops, rkeys, rvals, rres, back))

    def apply(self, ops: torch.Tensor, keys: torch.Tensor, vals: torch.Tensor, results: torch.Tensor) -> dict:
        """submit + results (synchronous convenience)."""
        return self.submit(ops, keys, vals, results).results()

    def submit_host(self, ops: torch.Tensor, keys: torch.Tensor, vals: torch.Tensor,
                    results: torch.Tensor) -> "ShardedTicket":
        """Host (pinned) slice buffers: H2D of the slice on the current stream, submit, D2H of the results;
        results are valid once the ticket's results() returns."""
        dev = self.device
        d = [torch.empty(x.shape, dtype=x.dtype, device=dev) for x in (ops, keys, vals)]
        for dst, src in zip(d, (ops, keys, vals)):
            dst.copy_(src, non_blocking=True)
        dres = torch.empty(results.shape, dtype=results.dtype, device=dev)
        t = self.submit(*d, dres)
        results.copy_(dres, non_blocking=True)
        t.keep = (t.keep, d, dres)
        return t

    def scan(self):
        return self.engine.scan()


class ShardedTicket:
    """A submitted global batch on this rank.  results() waits for the shard's batch and returns its stats
    with the GLOBAL status (the minimum over every shard's status, already all-reduced on the device)."""

    def __init__(self, sh: ShardedEirene, tk, status: torch.Tensor | None, n: int, keep=None,
                 rejected: int | None = None):
        self.sh, self.tk, self.status, self.n, self.keep = sh, tk, status, n, keep
        self.fixed = rejected

    def results(self) -> dict:
        if self.fixed is not None:   # rejected before any shard applied anything (invalid request)
            return {"rc": self.fixed, "status": self.fixed, "n": self.n, "launches": 0, "stage_ms": [0.0] * 8,
                    "device_ns": 0}
        st = {"rc": 0, "status": 0, "n": 0, "launches": 0, "stage_ms": [0.0] * 8, "device_ns": 0}
        if self.tk is not None:
            st = self.sh.engine.results(self.tk, raise_on_error=False)
        g = int(self.status.item())
        st["shard_status"] = st["status"]
        st["rc"] = st["status"] = g
        self.keep = None
        return st
