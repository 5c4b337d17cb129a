"""Key-range sharded Eirene over torch.distributed (one process per GPU).

SURVEY.md §8(e): requests on different keys are independent (§8(c)), so the
tree is partitioned by key range -- shard r owns [splitter[r-1], splitter[r]),
the splitters being equal-count quantiles of the bulk-loaded keys -- and each
batch needs one exchange step each way:

  1. every rank holds the contiguous timestamp slice r of the global batch;
  2. route_partition (CUDA kernel) stably groups the slice by destination
     shard (dest = upper_bound(splitters, key)) and counts per destination;
  3. all_to_all_single on the counts, an all_reduce of the validity flag;
  4. all_to_all_single on the payload (NCCL over NVLink 5 / NVSwitch);
     the receiver's concatenation in source-rank order is timestamp-ordered,
     so the shard's stable (key, ts) sort keeps linearizability (per-key
     locality of linearizability, Herlihy & Wing [17]);
  5. the shard runs the single-GPU hot path (eirene_submit_batch);
  6. all_to_all_single returns the results; route_unpermute (CUDA kernel)
     puts them back in the slice's timestamp order.

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
                 engine=None, router=None, **tree_kw):
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
        self.flag = torch.zeros(1, dtype=torch.int32, device=self.device)

    def apply(self, ops: torch.Tensor, keys: torch.Tensor, vals: torch.Tensor, results: torch.Tensor) -> dict:
        """Process this rank's timestamp slice of a global batch; results in slice order."""
        P = self.world
        sops, skeys, svals, perm, counts = self.router.route_partition(ops, keys, vals, self.splitters, P,
                                                                      invalid=self.flag)
        recv_counts = torch.empty_like(counts)
        if P > 1:
            dist.all_to_all_single(recv_counts, counts, group=self.group)
            dist.all_reduce(self.flag, op=dist.ReduceOp.MAX, group=self.group)
        else:
            recv_counts.copy_(counts)
        sc = counts.cpu().tolist()
        rc = recv_counts.cpu().tolist()
        invalid = int(self.flag.item())
        self.flag.zero_()
        if invalid:
            return {"rc": -1, "status": -1, "n": int(ops.numel()), "launches": 0, "stage_ms": [0.0] * 8}
        nrecv = int(sum(rc))
        dev = self.device
        rops = torch.empty(nrecv, dtype=torch.uint8, device=dev)
        rkeys = torch.empty(nrecv, dtype=torch.uint64, device=dev)
        rvals = torch.empty(nrecv, dtype=torch.uint64, device=dev)
        if P > 1:
            dist.all_to_all_single(_i64(rkeys), _i64(skeys), rc, sc, group=self.group)
            dist.all_to_all_single(_i64(rvals), _i64(svals), rc, sc, group=self.group)
            dist.all_to_all_single(rops, sops, rc, sc, group=self.group)
        else:
            rops.copy_(sops)
            rkeys.copy_(skeys)
            rvals.copy_(svals)
        rres = torch.empty(nrecv, dtype=torch.uint64, device=dev)
        st = {"rc": 0, "status": 0, "n": nrecv, "launches": 0, "stage_ms": [0.0] * 8}
        if nrecv:
            _, st = self.engine.apply(rops, rkeys, rvals, rres)
        back = torch.empty(int(sum(sc)), dtype=torch.uint64, device=dev)
        if P > 1:
            dist.all_to_all_single(_i64(back), _i64(rres), sc, rc, group=self.group)
        else:
            back.copy_(rres)
        self.router.route_unpermute(back, perm, out=results)
        return st

    def scan(self):
        return self.engine.scan()
