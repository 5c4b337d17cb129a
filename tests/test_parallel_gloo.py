"""Multi-process (world size 2, gloo, CPU) test of the key-range sharded path's
host logic (parallel.ShardedEirene): splitters, count exchange, concatenation
order of the all-to-all, inverse permutation, global-batch rejection.  The CUDA
per-shard engine and routing kernels are replaced by CPU stand-ins with the
same contract (the oracle as engine, numpy stable partition as router); the
CUDA routing kernels themselves are checked in tests/test_gpu_sharded.py."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

NF = 0xFFFFFFFFFFFFFFFF


class CpuRouter:
    """Stand-in for EireneTree.route_partition / route_unpermute (include/eirene.h contract)."""

    def route_partition(self, ops, keys, vals, splitters, P, invalid=None):
        k = keys.numpy()
        o = ops.numpy()
        v = vals.numpy()
        sp = splitters.numpy()[: P - 1]
        dest = np.searchsorted(sp, k, side="right") if P > 1 else np.zeros(k.size, np.int64)
        order = np.argsort(dest, kind="stable")
        counts = np.bincount(dest, minlength=P).astype(np.int32)
        if invalid is not None:
            up = (o == 1) | (o == 2)
            bad = (o > 3) | (k == np.uint64(NF)) | (up & (v == np.uint64(NF)))
            if bad.any():
                invalid.fill_(1)
        return (torch.from_numpy(o[order].copy()), torch.from_numpy(k[order].copy()),
                torch.from_numpy(v[order].copy()), torch.from_numpy(order.astype(np.int32)),
                torch.from_numpy(counts))

    def route_partition_packed(self, ops, keys, vals, splitters, P):
        o, k, v, perm, counts = self.route_partition(ops, keys, vals, splitters, P)
        bad = np.zeros(1, np.int32)
        self.route_partition(ops, keys, vals, splitters, P, invalid=torch.from_numpy(bad))
        rec = np.stack([k.numpy(), v.numpy(), o.numpy().astype(np.uint64)], axis=1).reshape(-1)
        c2 = np.stack([counts.numpy(), np.full(P, bad[0], np.int32)], axis=1).reshape(-1)
        return torch.from_numpy(rec.copy()), perm, torch.from_numpy(c2.astype(np.int32))

    def route_unpack(self, rec, n):
        r = rec.numpy().reshape(n, 3)
        return (torch.from_numpy(r[:, 2].astype(np.uint8)), torch.from_numpy(r[:, 0].copy()),
                torch.from_numpy(r[:, 1].copy()))

    def route_unpermute(self, back, perm, out=None):
        res = np.empty(back.numel(), np.uint64)
        res[perm.numpy()] = back.numpy()
        if out is None:
            return torch.from_numpy(res)
        out.copy_(torch.from_numpy(res))
        return out


class OracleEngine:
    """Stand-in for EireneTree (per-shard single-GPU path) built on the CPU oracle."""

    def __init__(self):
        import oracle
        self.m = oracle.MapOracle()

    def bulk_load(self, keys, vals):
        self.m.load(keys.numpy(), vals.numpy())

    def apply(self, ops, keys, vals, results):
        r = self.m.apply(ops.numpy(), keys.numpy(), vals.numpy())
        results.copy_(torch.from_numpy(r))
        return results, {"rc": 0, "status": 0, "n": int(ops.numel()), "launches": 0, "stage_ms": [0.0] * 8}

    def submit(self, ops, keys, vals, results):
        self.apply(ops, keys, vals, results)
        return 1

    def status_async(self, tk, out):
        out.fill_(0)
        return out

    def results(self, tk, raise_on_error=True):
        return {"rc": 0, "status": 0, "n": 0, "launches": 0, "stage_ms": [0.0] * 8}

    def scan(self):
        k, v = self.m.scan()
        return torch.from_numpy(k), torch.from_numpy(v)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, outdir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W
        from paper_conf_ppopp_zhangz0lzl23_b200.parallel import ShardedEirene
        w = W.Workload(2, tree=1 << 12, batch=world * 1024,
                       fracs={W.QUERY: 0.5, W.UPDATE: 0.2, W.INSERT: 0.2, W.DELETE: 0.1})
        sh = ShardedEirene(w.keys, w.vals, max_batch=1024, device="cpu", engine=OracleEngine(), router=CpuRouter())
        ref = oracle.MapOracle()
        ref.load(w.keys, w.vals)
        bad = 0
        for b in range(4):
            ops, keys, vals = w.batch_arrays(b)
            want = ref.apply(ops, keys, vals)
            sl = slice(rank * 1024, (rank + 1) * 1024)
            res = torch.empty(1024, dtype=torch.uint64)
            st = sh.apply(torch.from_numpy(ops[sl].copy()), torch.from_numpy(keys[sl].copy()),
                          torch.from_numpy(vals[sl].copy()), res)
            assert st["status"] == 0
            bad += int(np.sum(res.numpy() != want[sl]))
        # the shard holds exactly the oracle's final state restricted to its key range
        k, v = sh.scan()
        rk, rv = ref.scan()
        sel = (rk >= np.uint64(sh.lo)) & ((rk < np.uint64(sh.hi)) if sh.hi != NF else True)
        same = np.array_equal(k.numpy(), rk[sel]) and np.array_equal(v.numpy(), rv[sel])
        # a bad request on ONE rank rejects the global batch on every rank (no shard applies)
        ops, keys, vals = w.batch_arrays(9)
        sl = slice(rank * 1024, (rank + 1) * 1024)
        o = ops[sl].copy()
        if rank == 1:
            o[5] = 7
        st = sh.apply(torch.from_numpy(o), torch.from_numpy(keys[sl].copy()), torch.from_numpy(vals[sl].copy()),
                      torch.empty(1024, dtype=torch.uint64))
        k2, v2 = sh.scan()
        untouched = np.array_equal(k2.numpy(), k.numpy()) and np.array_equal(v2.numpy(), v.numpy())
        with open(os.path.join(outdir, f"r{rank}.txt"), "w") as f:
            f.write(f"{bad} {int(same)} {st['status']} {int(untouched)}\n")
    finally:
        dist.destroy_process_group()


def test_sharded_two_ranks_gloo():
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(world, _free_port(), d), nprocs=world, join=True)
        for r in range(world):
            bad, same, st, untouched = open(os.path.join(d, f"r{r}.txt")).read().split()
            assert bad == "0", f"rank {r}: {bad} results differ from the oracle"
            assert same == "1", f"rank {r}: shard contents differ from the oracle"
            assert st == "-1" and untouched == "1", f"rank {r}: invalid global batch not rejected everywhere"


def test_splitters_partition_keys():
    from paper_conf_ppopp_zhangz0lzl23_b200.parallel import shard_range, splitters_for
    keys = np.arange(0, 1000, 3, dtype=np.uint64)
    for P in (1, 2, 3, 8):
        sp = splitters_for(keys, P)
        assert sp.size == P - 1 and np.all(np.diff(sp.astype(np.int64)) > 0)
        counts = [np.sum((keys >= np.uint64(lo)) & ((keys < np.uint64(hi)) if hi != NF else True))
                  for lo, hi in (shard_range(sp, r, P) for r in range(P))]
        assert sum(counts) == keys.size and max(counts) - min(counts) <= 1
