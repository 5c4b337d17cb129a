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


class OracleArenaEngine(OracleEngine):
    """OracleEngine plus a CPU stand-in of the fused-routing arena calls (include/eirene.h contract): each rank's
    arena is a POSIX shared-memory segment {P x (count, invalid, start, epoch) u32, cap result u64, P x cap x 3
    record u64}; its name plays the IPC handle, so the peers' "pushes" are plain stores into it."""

    def __init__(self):
        super().__init__()
        self.views = {}
        self.shms = []
        self.epoch = 0

    def _view(self, shm, P, cap):
        buf = shm.buf
        cnt = np.ndarray((P, 4), np.uint32, buf, 0)
        res = np.ndarray((cap,), np.uint64, buf, 1024)
        rec = np.ndarray((P, cap, 3), np.uint64, buf, 1024 + 8 * cap)
        return cnt, res, rec

    def route_arena_create(self, P, rank, cap):
        from multiprocessing import shared_memory
        shm = shared_memory.SharedMemory(create=True, size=1024 + 8 * cap + 24 * P * cap)
        self.shms.append(shm)
        self.P, self.me, self.cap = P, rank, cap
        np.ndarray((1024,), np.uint8, shm.buf, 0)[:] = 0
        key = len(self.views) + 1
        self.views[key] = self._view(shm, P, cap)
        return key, shm.name.encode().ljust(64, b"\0")

    def route_arena_open_ipc(self, handle):
        from multiprocessing import shared_memory
        shm = shared_memory.SharedMemory(name=handle.rstrip(b"\0").decode())
        self.shms.append(shm)
        key = len(self.views) + 1
        self.views[key] = self._view(shm, self.P, self.cap)
        return key

    def route_arena_connect(self, addrs):
        self.peers = [self.views[a] for a in addrs]
        self.own = self.peers[self.me]

    def route_push(self, ops, keys, vals, splitters, perm):
        P = self.P
        o, k, v, pm, counts = CpuRouter().route_partition(ops, keys, vals, splitters, P)
        bad = np.zeros(1, np.int32)
        CpuRouter().route_partition(ops, keys, vals, splitters, P, invalid=torch.from_numpy(bad))
        perm.copy_(pm)
        self.epoch += 1
        start = np.concatenate([[0], np.cumsum(counts.numpy())])
        for d in range(P):
            c = int(counts[d])
            rec = self.peers[d][2]
            rec[self.me, :c, 0] = k.numpy()[start[d]:start[d] + c]
            rec[self.me, :c, 1] = v.numpy()[start[d]:start[d] + c]
            rec[self.me, :c, 2] = o.numpy()[start[d]:start[d] + c]
            self.peers[d][0][self.me] = (c, bad[0], start[d], self.epoch)

    def route_pull(self, ops, keys, vals):
        cnt, _, rec = self.own
        assert np.all(cnt[:, 3] == self.epoch), "a peer's push never arrived"
        if cnt[:, 1].any():
            return int(cnt[:, 0].sum()), 1
        parts = [rec[s, :cnt[s, 0]] for s in range(self.P)]
        r = np.concatenate(parts) if parts else np.zeros((0, 3), np.uint64)
        n = r.shape[0]
        keys[:n].copy_(torch.from_numpy(r[:, 0].copy()))
        vals[:n].copy_(torch.from_numpy(r[:, 1].copy()))
        ops[:n].copy_(torch.from_numpy(r[:, 2].astype(np.uint8)))
        return n, 0

    def route_push_results(self, results):
        cnt = self.own[0]
        off = 0
        for s in range(self.P):
            c, st = int(cnt[s, 0]), int(cnt[s, 2])
            self.peers[s][1][st:st + c] = results.numpy()[off:off + c]
            off += c

    def route_unpermute_arena(self, perm, out):
        res = np.empty(perm.numel(), np.uint64)
        res[perm.numpy()] = self.own[1][:perm.numel()]
        out.copy_(torch.from_numpy(res))
        return out

    def close_arenas(self):
        for shm in self.shms[1:]:
            shm.close()
        if self.shms:
            self.shms[0].close()
            self.shms[0].unlink()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, outdir, fused=False):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W
        from paper_conf_ppopp_zhangz0lzl23_b200.parallel import ShardedEirene
        w = W.Workload(2, tree=1 << 12, batch=world * 1024,
                       fracs={W.QUERY: 0.5, W.UPDATE: 0.2, W.INSERT: 0.2, W.DELETE: 0.1})
        eng = OracleArenaEngine() if fused else OracleEngine()
        sh = ShardedEirene(w.keys, w.vals, max_batch=1024, device="cpu", engine=eng, router=CpuRouter(), fused=fused)
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
        dist.barrier()
        if fused:
            eng.close_arenas()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("fused", [False, True])
def test_sharded_two_ranks_gloo(fused):
    """fused=True: the fused push over the ranks' arenas (ShardedEirene._submit_fused: push, barrier, pull,
    shard batch, results pushed back, status all-reduce as the second barrier, unpermute)."""
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(world, _free_port(), d, fused), nprocs=world, join=True)
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
