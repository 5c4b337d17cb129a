"""GPU test of the key-range sharded path on ONE device: P shard trees, the CUDA
routing kernels (eirene_route_partition / eirene_route_unpermute), and the
all-to-all emulated by concatenating per-destination segments in source-rank
order (exactly what all_to_all_single delivers).  Results must be bit-exact
with the oracle on the global batch and identical for every P."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W
from paper_conf_ppopp_zhangz0lzl23_b200.parallel import shard_range, splitters_for

pytestmark = pytest.mark.gpu
NF = 0xFFFFFFFFFFFFFFFF


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    torch.cuda.set_device(0)
    return torch.device("cuda", 0)


def run_sharded(dev, w, P, nb, per_rank, packed=False):
    from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree
    sp = splitters_for(w.keys, P)
    sp_t = torch.from_numpy(sp if P > 1 else np.zeros(1, np.uint64)).to(dev)
    trees = []
    for r in range(P):
        lo, hi = shard_range(sp, r, P)
        sel = (w.keys >= np.uint64(lo)) & ((w.keys < np.uint64(hi)) if hi != NF else True)
        t = EireneTree(max_keys=1 << 18, max_batch=P * per_rank, key_lo=lo, key_hi=hi)
        if sel.any():
            t.bulk_load(torch.from_numpy(w.keys[sel].copy()).to(dev), torch.from_numpy(w.vals[sel].copy()).to(dev))
        trees.append(t)
    out = []
    for b in range(nb):
        ops, keys, vals = w.batch_arrays(b)
        routed = []
        for r in range(P):     # every source rank partitions its ts-slice
            sl = slice(r * per_rank, (r + 1) * per_rank)
            args = (torch.from_numpy(ops[sl].copy()).to(dev), torch.from_numpy(keys[sl].copy()).to(dev),
                    torch.from_numpy(vals[sl].copy()).to(dev), sp_t, P)
            if packed:   # 24 B records + (count, validity flag) per destination, unpacked after the "exchange"
                rec, perm, cnt2 = trees[r].route_partition_packed(*args)
                c2 = cnt2.cpu().numpy()
                c = c2[0::2]
                assert np.all(c2[1::2] == 0)
                so, sk, sv = trees[r].route_unpack(rec, int(c.sum()))
            else:
                so, sk, sv, perm, cnt = trees[r].route_partition(*args)
                c = cnt.cpu().numpy()
            off = np.concatenate([[0], np.cumsum(c)])
            routed.append((so, sk, sv, perm, off))
        back = [[None] * P for _ in range(P)]
        for d in range(P):      # destination shard: concatenation in source-rank order
            o = torch.cat([routed[r][0][routed[r][4][d]:routed[r][4][d + 1]] for r in range(P)])
            k = torch.cat([routed[r][1][routed[r][4][d]:routed[r][4][d + 1]] for r in range(P)])
            v = torch.cat([routed[r][2][routed[r][4][d]:routed[r][4][d + 1]] for r in range(P)])
            res = torch.empty(o.numel(), dtype=torch.uint64, device=dev)
            if o.numel():
                trees[d].apply(o, k, v, res)
            pos = 0
            for r in range(P):
                m = int(routed[r][4][d + 1] - routed[r][4][d])
                back[r][d] = res[pos:pos + m]
                pos += m
        full = []
        for r in range(P):      # reverse exchange + inverse permutation
            recv = torch.cat([back[r][d] for d in range(P)])
            full.append(trees[r].route_unpermute(recv, routed[r][3]).cpu().numpy())
        out.append(np.concatenate(full))
    scans = [t.scan() for t in trees]
    keys = np.concatenate([s[0].cpu().numpy() for s in scans])
    vals = np.concatenate([s[1].cpu().numpy() for s in scans])
    return out, keys, vals


@pytest.mark.parametrize("packed", [False, True])
@pytest.mark.parametrize("cfg", [2, 3])
def test_sharded_equals_oracle_for_every_P(dev, cfg, packed):
    per_rank = 4096
    nb = 3
    results = {}
    for P in (1, 2, 4, 8):
        w = W.Workload(cfg, tree=1 << 16, batch=P * per_rank,
                       fracs={W.QUERY: 0.5, W.UPDATE: 0.3, W.INSERT: 0.15, W.DELETE: 0.05})
        ref = oracle.MapOracle()
        ref.load(w.keys, w.vals)
        out, k, v = run_sharded(dev, w, P, nb, per_rank, packed)
        # replay the same batches on the oracle (a fresh generator: the batch
        # stream is a pure function of (cfg, seed, batch index))
        w2 = W.Workload(cfg, tree=1 << 16, batch=P * per_rank,
                        fracs={W.QUERY: 0.5, W.UPDATE: 0.3, W.INSERT: 0.15, W.DELETE: 0.05})
        for b in range(nb):
            ops, keys, vals = w2.batch_arrays(b)
            want = ref.apply(ops, keys, vals)
            assert np.array_equal(out[b], want), f"P={P} batch {b}: {int(np.sum(out[b] != want))} differ"
        rk, rv = ref.scan()
        assert np.array_equal(k, rk) and np.array_equal(v, rv), f"P={P}: final state differs"
        results[P] = out


def test_packed_partition_flags_invalid_slice(dev):
    """route_partition_packed: one invalid request in the slice sets the validity
    word of every destination (so one exchange tells every rank), counts intact."""
    from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree
    t = EireneTree(max_keys=1 << 12, max_batch=1 << 12)
    rng = np.random.default_rng(3)
    n, P = 3000, 4
    ops = rng.integers(0, 4, n).astype(np.uint8)
    keys = rng.integers(1, 1 << 62, n, dtype=np.uint64)
    vals = rng.integers(0, 1 << 62, n, dtype=np.uint64)
    sp = np.sort(rng.integers(1, 1 << 62, P - 1, dtype=np.uint64))
    sp_t = torch.from_numpy(sp).to(dev)
    for bad in (False, True):
        o = ops.copy()
        if bad:
            o[1234] = 9
        rec, perm, cnt2 = t.route_partition_packed(torch.from_numpy(o).to(dev), torch.from_numpy(keys).to(dev),
                                                   torch.from_numpy(vals).to(dev), sp_t, P)
        c2 = cnt2.cpu().numpy()
        dest = np.searchsorted(sp, keys, side="right")
        assert np.array_equal(c2[0::2], np.bincount(dest, minlength=P))
        assert np.all(c2[1::2] == (1 if bad else 0))
        r = rec.cpu().numpy().reshape(n, 3)
        pm = perm.cpu().numpy()
        assert np.array_equal(r[:, 0], keys[pm]) and np.array_equal(r[:, 1], vals[pm])
        assert np.array_equal(r[:, 2], o[pm].astype(np.uint64))
        assert np.all(np.diff(dest[pm]) >= 0)                       # grouped by destination
        for d in range(P):                                           # stable: timestamp order inside
            assert np.all(np.diff(pm[dest[pm] == d]) > 0)
    t.close()


def fused_shards(dev, w, P, per_rank):
    """P shard trees with connected receive arenas (one process: the peers' arenas are plain device pointers)."""
    from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree
    sp = splitters_for(w.keys, P)
    sp_t = torch.from_numpy(sp if P > 1 else np.zeros(1, np.uint64)).to(dev)
    trees, addrs = [], []
    for r in range(P):
        lo, hi = shard_range(sp, r, P)
        sel = (w.keys >= np.uint64(lo)) & ((w.keys < np.uint64(hi)) if hi != NF else True)
        t = EireneTree(max_keys=1 << 18, max_batch=P * per_rank, key_lo=lo, key_hi=hi)
        if sel.any():
            t.bulk_load(torch.from_numpy(w.keys[sel].copy()).to(dev), torch.from_numpy(w.vals[sel].copy()).to(dev))
        addrs.append(t.route_arena_create(P, r, per_rank)[0])
        trees.append(t)
    for t in trees:
        t.route_arena_connect(addrs)
    return trees, sp_t


def fused_batch(dev, trees, sp_t, P, per_rank, ops, keys, vals):
    """One global batch through the fused push: every source pushes, every shard pulls / applies / pushes
    its results back, every source unpermutes from its arena (one stream: program order is the barrier)."""
    perms = []
    for r in range(P):
        sl = slice(r * per_rank, (r + 1) * per_rank)
        perm = torch.empty(sl.stop - sl.start, dtype=torch.int32, device=dev)
        trees[r].route_push(torch.from_numpy(ops[sl].copy()).to(dev), torch.from_numpy(keys[sl].copy()).to(dev),
                            torch.from_numpy(vals[sl].copy()).to(dev), sp_t, perm)
        perms.append(perm)
    flags = []
    for d in range(P):
        cap = P * per_rank
        o = torch.empty(cap, dtype=torch.uint8, device=dev)
        k = torch.empty(cap, dtype=torch.uint64, device=dev)
        v = torch.empty(cap, dtype=torch.uint64, device=dev)
        n, inv = trees[d].route_pull(o, k, v)
        flags.append(inv)
        res = torch.empty(max(n, 1), dtype=torch.uint64, device=dev)
        if n and not inv:
            trees[d].apply(o[:n], k[:n], v[:n], res[:n])
        trees[d].route_push_results(res)
    out = []
    for r in range(P):
        res = torch.empty(per_rank, dtype=torch.uint64, device=dev)
        out.append(trees[r].route_unpermute_arena(perms[r], res).cpu().numpy())
    return np.concatenate(out), flags


@pytest.mark.parametrize("cfg", [2, 3])
def test_fused_push_equals_oracle_for_every_P(dev, cfg):
    """Fused routing (eirene_route_push / pull / push_results / unpermute_arena):
    bit-exact with the oracle on every global batch and the final state, for P in {1, 2, 4, 8}."""
    per_rank = 4096
    nb = 3
    fr = {W.QUERY: 0.5, W.UPDATE: 0.3, W.INSERT: 0.15, W.DELETE: 0.05}
    for P in (1, 2, 4, 8):
        w = W.Workload(cfg, tree=1 << 16, batch=P * per_rank, fracs=fr)
        ref = oracle.MapOracle()
        ref.load(w.keys, w.vals)
        trees, sp_t = fused_shards(dev, w, P, per_rank)
        for b in range(nb):
            ops, keys, vals = w.batch_arrays(b)
            got, flags = fused_batch(dev, trees, sp_t, P, per_rank, ops, keys, vals)
            assert flags == [0] * P
            want = ref.apply(ops, keys, vals)
            assert np.array_equal(got, want), f"P={P} batch {b}: {int(np.sum(got != want))} differ"
        scans = [t.scan() for t in trees]
        k = np.concatenate([s[0].cpu().numpy() for s in scans])
        v = np.concatenate([s[1].cpu().numpy() for s in scans])
        rk, rv = ref.scan()
        assert np.array_equal(k, rk) and np.array_equal(v, rv), f"P={P}: final state differs"
        for t in trees:
            t.close()


def test_fused_push_invalid_slice_and_missing_push(dev):
    """One invalid request in one source's slice: every shard's pull reports it (the global batch is
    rejected everywhere, no shard applies); a source that skips its push makes every pull fail (EINTERNAL)."""
    from paper_conf_ppopp_zhangz0lzl23_b200 import _ffi
    P, per_rank = 4, 2048
    w = W.Workload(2, tree=1 << 14, batch=P * per_rank)
    trees, sp_t = fused_shards(dev, w, P, per_rank)
    ops, keys, vals = w.batch_arrays(0)
    ops = ops.copy()
    ops[per_rank + 77] = 9   # rank 1's slice
    _, flags = fused_batch(dev, trees, sp_t, P, per_rank, ops, keys, vals)
    assert flags == [1] * P
    ops, keys, vals = w.batch_arrays(1)
    for r in range(1, P):    # rank 0 never pushes this batch
        sl = slice(r * per_rank, (r + 1) * per_rank)
        perm = torch.empty(per_rank, dtype=torch.int32, device=dev)
        trees[r].route_push(torch.from_numpy(ops[sl].copy()).to(dev), torch.from_numpy(keys[sl].copy()).to(dev),
                            torch.from_numpy(vals[sl].copy()).to(dev), sp_t, perm)
    o = torch.empty(P * per_rank, dtype=torch.uint8, device=dev)
    k = torch.empty(P * per_rank, dtype=torch.uint64, device=dev)
    for d in range(1, P):
        with pytest.raises(RuntimeError, match="EINTERNAL|watchdog|internal"):
            trees[d].route_pull(o, k, k.clone())
    assert _ffi.EIRENE_IPC_HANDLE_BYTES == 64
    for t in trees:
        t.close()
