"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by
element, bit-exact (integer path).  Run with -m gpu on a B200."""
import json
import os

import numpy as np
import pytest
import torch

import oracle
from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W

pytestmark = pytest.mark.gpu

NF = np.uint64(0xFFFFFFFFFFFFFFFF)


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ppopp_zhangz0lzl23_b200.build import build
    build()
    torch.cuda.set_device(0)
    return torch.device("cuda", 0)


def T(a, dev):
    return torch.from_numpy(np.ascontiguousarray(a)).to(dev)


def make_tree(dev, keys, vals, max_keys=None, max_batch=1 << 16, fill=1.0, **kw):
    from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree
    t = EireneTree(max_keys=max_keys or max(1 << 12, 4 * len(keys)), max_batch=max_batch, **kw)
    if len(keys):
        t.bulk_load(T(keys, dev), T(vals, dev), leaf_fill=fill)
    return t


def run_and_compare(t, ref, ops, keys, vals, dev, check_scan=True):
    res, st = t.apply(T(ops, dev), T(keys, dev), T(vals, dev))
    want = ref.apply(ops, keys, vals)
    got = res.cpu().numpy()
    bad = np.nonzero(got != want)[0]
    assert bad.size == 0, (f"{bad.size} of {len(ops)} results differ; first at {bad[:5]}: "
                           f"got {got[bad[:5]]}, want {want[bad[:5]]}, ops {ops[bad[:5]]}")
    if check_scan:
        k, v = t.scan()
        rk, rv = ref.scan()
        assert np.array_equal(k.cpu().numpy(), rk), "scan keys differ"
        assert np.array_equal(v.cpu().numpy(), rv), "scan values differ"
    return st


def _rand_keys(rng, n, hi=1 << 40):
    k = np.unique(rng.integers(1, hi, size=2 * n + 8, dtype=np.uint64))[:n]
    return k, rng.integers(0, 1 << 62, size=k.size, dtype=np.uint64)


@pytest.mark.parametrize("n,fill", [(1, 1.0), (15, 1.0), (16, 1.0), (17, 1.0), (1000, 1.0), (1000, 0.5),
                                    (100000, 0.7), (70000, 0.01)])
def test_bulk_load_scan_roundtrip(dev, n, fill):
    rng = np.random.default_rng(n)
    keys, vals = _rand_keys(rng, n)
    t = make_tree(dev, keys, vals, fill=fill)
    k, v = t.scan()
    assert np.array_equal(k.cpu().numpy(), keys) and np.array_equal(v.cpu().numpy(), vals)
    rc, nk = t.check_invariants()
    assert rc == 0 and nk == n
    # sub-range scans are inclusive on both ends
    lo, hi = int(keys[n // 3]), int(keys[(2 * n) // 3])
    k, v = t.scan(lo, hi)
    sel = (keys >= lo) & (keys <= hi)
    assert np.array_equal(k.cpu().numpy(), keys[sel])


def test_bulk_load_rejects_bad_keys(dev):
    from paper_conf_ppopp_zhangz0lzl23_b200._ffi import EireneError
    t = make_tree(dev, np.empty(0, np.uint64), np.empty(0, np.uint64))
    with pytest.raises(EireneError):
        t.bulk_load(T(np.array([5, 3], np.uint64), dev), T(np.array([1, 2], np.uint64), dev))
    t2 = make_tree(dev, np.empty(0, np.uint64), np.empty(0, np.uint64))
    with pytest.raises(EireneError):
        t2.bulk_load(T(np.array([5, 5], np.uint64), dev), T(np.array([1, 2], np.uint64), dev))


def test_fig3_worked_example(dev, golden_dir):
    with open(os.path.join(golden_dir, "fig3.json")) as f:
        g = json.load(f)
    val = g["values"]
    opc = {"Q": 0, "U": 1, "I": 2, "D": 3}
    pk = np.array([k for k, _ in g["pre_batch"]], np.uint64)
    pv = np.array([val[v] for _, v in g["pre_batch"]], np.uint64)
    reqs = sorted(g["requests"], key=lambda r: r["ts"])
    ops = np.array([opc[r["op"]] for r in reqs], np.uint8)
    keys = np.array([r["key"] for r in reqs], np.uint64)
    vals = np.array([val[r["val"]] if "val" in r else 0 for r in reqs], np.uint64)
    t = make_tree(dev, pk, pv)
    res, st = t.apply(T(ops, dev), T(keys, dev), T(vals, dev))
    got = res.cpu().numpy()
    for part in ("expected_results_paper", "expected_results_reading1"):
        for ts, v in g[part].items():
            if not ts.startswith("_"):
                assert int(got[int(ts) - 1]) == val[v], (ts, int(got[int(ts) - 1]))
    assert st["distinct"] == 3 and st["issued_w"] == 2 and st["issued_q"] == 1
    k, v = t.scan()
    assert [(int(a), int(b)) for a, b in zip(k.cpu(), v.cpu())] == [(kk, val[vv]) for kk, vv in g["final_state"]]


def test_query_only(dev):
    rng = np.random.default_rng(3)
    keys, vals = _rand_keys(rng, 50000)
    t = make_tree(dev, keys, vals)
    ref = oracle.MapOracle(); ref.load(keys, vals)
    q = np.concatenate([keys[rng.integers(0, keys.size, 30000)], rng.integers(1, 1 << 40, 20000, dtype=np.uint64)])
    rng.shuffle(q)
    st = run_and_compare(t, ref, np.zeros(q.size, np.uint8), q, np.zeros(q.size, np.uint64), dev)
    assert st["issued_w"] == 0 and st["distinct"] == np.unique(q).size


@pytest.mark.parametrize("cfg", [2, 3])
def test_read_update_mixes_small(dev, cfg):
    """cfg2 (95/5 uniform) and cfg3 (50/50 Zipf) shapes at reduced size, several batches."""
    w = W.Workload(cfg, tree=1 << 16, batch=1 << 15)
    t = make_tree(dev, w.keys, w.vals, max_batch=1 << 15)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    for b in range(4):
        ops, keys, vals = w.batch_arrays(b)
        st = run_and_compare(t, ref, ops, keys, vals, dev, check_scan=(b == 3))
        assert st["leaf_splits"] == 0 and st["new_leaves"] == 0
    assert t.check_invariants()[0] == 0


def test_cfg1_inserts_split_every_leaf(dev):
    """cfg1 at full size: 2^16-key tree, one 2^16 batch of 50% query / 50% insert."""
    w = W.Workload(1)
    t = make_tree(dev, w.keys, w.vals, max_batch=1 << 16)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    ops, keys, vals = w.batch_arrays(0)
    st = run_and_compare(t, ref, ops, keys, vals, dev)
    assert st["leaf_splits"] > 0.99 * 4096
    rc, nk = t.check_invariants()
    assert rc == 0 and nk == ref.size()


def test_cfg4_full_size_growth(dev):
    """cfg4 at full size, as the bench runs it: a 2^20-key tree grown by four 2^20-request batches of 90% insert /
    10% delete (toward 2^22 keys: split storms on every batch, level-synchronous propagation, batched leaf runs);
    every result and the final scan bit-exact, invariants intact."""
    w = W.Workload(4)
    C = W.CONFIGS[4]
    t = make_tree(dev, w.keys, w.vals, max_keys=C["tree"] + C["per_tree"] * C["batch"] + (1 << 12),
                  max_batch=C["batch"])
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    splits = 0
    for b in range(C["per_tree"]):
        ops, keys, vals = w.batch_arrays(b)
        st = run_and_compare(t, ref, ops, keys, vals, dev, check_scan=b + 1 == C["per_tree"])
        splits += st["leaf_splits"]
    assert splits > C["batch"] // 8   # (the storm did happen)
    rc, nk = t.check_invariants()
    assert rc == 0 and nk == ref.size()
    t.close()


@pytest.mark.parametrize("regroup", [True, False])
@pytest.mark.parametrize("threshold,force", [(4, False), (0, False), (1, False), (1 << 30, False), (4, True)])
def test_structural_mix_threshold_and_regroup(dev, regroup, threshold, force):
    """Inserts/deletes with splits; results identical for every THRESHOLD, FORCE_STM and
    regroup setting (metamorphic, SURVEY §8(c) readings 16-17)."""
    rng = np.random.default_rng(17)
    keys, vals = _rand_keys(rng, 3000, hi=1 << 20)
    t = make_tree(dev, keys, vals, max_batch=1 << 14, retry_threshold=threshold, force_stm=force,
                  regroup=regroup)
    ref = oracle.MapOracle(); ref.load(keys, vals)
    for b in range(5):
        n = 1 << 13
        ops = rng.choice(np.array([0, 1, 2, 3], np.uint8), n, p=[0.3, 0.2, 0.4, 0.1])
        ks = np.where(rng.random(n) < 0.5, keys[rng.integers(0, keys.size, n)],
                      rng.integers(1, 1 << 20, n, dtype=np.uint64)).astype(np.uint64)
        vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
        st = run_and_compare(t, ref, ops, ks, vs, dev, check_scan=True)
        if force or threshold == 0:
            assert st["stm_fallbacks"] > 0
    rc, nk = t.check_invariants()
    assert rc == 0 and nk == ref.size()


def test_single_key_storm(dev):
    """Every request on one key (the largest possible combine segment)."""
    rng = np.random.default_rng(5)
    keys, vals = _rand_keys(rng, 100)
    t = make_tree(dev, keys, vals, max_batch=1 << 16)
    ref = oracle.MapOracle(); ref.load(keys, vals)
    n = 1 << 16
    ops = rng.integers(0, 4, n).astype(np.uint8)
    ks = np.full(n, keys[7], np.uint64)
    vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
    st = run_and_compare(t, ref, ops, ks, vs, dev)
    assert st["distinct"] == 1


@pytest.mark.parametrize("seed", [0, 1])
def test_hot_key_groups(dev, seed):
    """Skewed batch over the full 64-bit key space: keys with 9000 (more than one
    group's shared-memory capacity), 5000 + 4000 (two hot keys, one oversized
    group if they share a bin), 300 and 40 copies, among uniform keys.  Covers
    the oversized-group L2 sort, the timestamp-stable slow path and the
    rank-placement fast path of the group sort (group.cu)."""
    rng = np.random.default_rng(40 + seed)
    keys, vals = _rand_keys(rng, 20000, hi=1 << 63)
    t = make_tree(dev, keys, vals, max_batch=1 << 16)
    ref = oracle.MapOracle(); ref.load(keys, vals)
    n = 1 << 16
    hot = [(keys[3], 9000), (keys[11], 5000), (keys[11] + np.uint64(1), 4000), (keys[20], 300),
           (keys[21], 40), (rng.integers(1, 1 << 63, dtype=np.uint64), 500)]
    parts = [np.full(c, k, np.uint64) for k, c in hot]
    rest = n - sum(c for _, c in hot)
    parts.append(np.where(rng.random(rest) < 0.5, rng.choice(keys, rest),
                          rng.integers(1, 1 << 63, rest, dtype=np.uint64)).astype(np.uint64))
    ks = np.concatenate(parts)
    rng.shuffle(ks)
    ops = rng.integers(0, 4, n).astype(np.uint8)
    vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
    run_and_compare(t, ref, ops, ks, vs, dev)
    # and a second batch on the grown tree
    ops2 = rng.integers(0, 4, n).astype(np.uint8)
    rng.shuffle(ks)
    run_and_compare(t, ref, ops2, ks, vs, dev)
    assert t.check_invariants()[0] == 0


def test_dense_key_range(dev):
    """Dense small integer keys: every request falls in the first bin, so one
    group holds the whole batch (oversized, many distinct keys: the generic
    L2 radix path)."""
    rng = np.random.default_rng(9)
    keys = np.arange(1, 20001, dtype=np.uint64)
    vals = rng.integers(0, 1 << 62, keys.size, dtype=np.uint64)
    t = make_tree(dev, keys, vals, max_batch=1 << 15)
    ref = oracle.MapOracle(); ref.load(keys, vals)
    n = 1 << 15
    ops = rng.integers(0, 4, n).astype(np.uint8)
    ks = rng.integers(1, 30000, n, dtype=np.uint64)
    vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
    run_and_compare(t, ref, ops, ks, vs, dev)
    assert t.check_invariants()[0] == 0


def test_tiny_tree_root_splits(dev):
    """Start from an empty tree (root is a leaf) and grow it by inserts: root splits."""
    rng = np.random.default_rng(8)
    t = make_tree(dev, np.empty(0, np.uint64), np.empty(0, np.uint64), max_keys=1 << 16, max_batch=4096)
    ref = oracle.MapOracle()
    for b, n in enumerate([1, 5, 16, 17, 300, 4096, 4096]):
        ops = rng.choice(np.array([0, 2, 3], np.uint8), n, p=[0.2, 0.7, 0.1])
        ks = rng.integers(1, 1 << 16, n, dtype=np.uint64)
        vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
        run_and_compare(t, ref, ops, ks, vs, dev)
        assert t.check_invariants()[0] == 0
    assert t.info()["height"] >= 3


def test_exhaustive_tiny_alphabet_key_tiled(dev):
    """Every sequence of length <= 4 over {Q, U(a), U(b), I(a), D} on one key, from
    both initial presence states, each placed on its own key: one GPU batch."""
    import itertools
    alphabet = [(0, 0), (1, 7), (1, 8), (2, 7), (3, 0)]
    seqs = [s for L in range(1, 5) for s in itertools.product(alphabet, repeat=L)]
    ops, keys, vals, pre_k, pre_v = [], [], [], [], []
    kid = 2
    for present in (False, True):
        for s in seqs:
            if present:
                pre_k.append(kid); pre_v.append(1000 + kid)
            for o, v in s:
                ops.append(o); keys.append(kid); vals.append(v)
            kid += 2
    ops = np.array(ops, np.uint8); keys = np.array(keys, np.uint64); vals = np.array(vals, np.uint64)
    # interleave the per-key sequences randomly, keeping each key's internal order:
    # random priorities, re-assigned in sorted order within each key
    rng = np.random.default_rng(0)
    prio = rng.random(keys.size)
    _, inv = np.unique(keys, return_inverse=True)
    grp = np.argsort(inv, kind="stable")
    bounds = np.flatnonzero(np.diff(inv[grp])) + 1
    for g in np.split(grp, bounds):
        prio[g] = np.sort(prio[g])
    order = np.argsort(prio)
    ops, keys, vals = ops[order], keys[order], vals[order]
    pre_k = np.array(pre_k, np.uint64); pre_v = np.array(pre_v, np.uint64)
    t = make_tree(dev, pre_k, pre_v, max_batch=1 << 17, max_keys=1 << 17)
    ref = oracle.MapOracle(); ref.load(pre_k, pre_v)
    run_and_compare(t, ref, ops, keys, vals, dev)


def test_invalid_batch_leaves_tree_untouched(dev):
    rng = np.random.default_rng(4)
    keys, vals = _rand_keys(rng, 1000)
    t = make_tree(dev, keys, vals)
    for bad in ("op", "key", "val"):
        ops = np.zeros(100, np.uint8); ops[:50] = 2
        ks = rng.integers(1, 1 << 40, 100, dtype=np.uint64)
        vs = rng.integers(0, 1 << 62, 100, dtype=np.uint64)
        if bad == "op":
            ops[77] = 9
        elif bad == "key":
            ks[3] = NF
        else:
            vs[10] = NF
        res = torch.empty(100, dtype=torch.uint64, device=dev)
        tk = t.submit(T(ops, dev), T(ks, dev), T(vs, dev), res)
        st = t.results(tk, raise_on_error=False)
        assert st["rc"] == -1 and st["status"] == -1
    k, v = t.scan()
    assert np.array_equal(k.cpu().numpy(), keys) and np.array_equal(v.cpu().numpy(), vals)


def test_delete_of_value_max_is_valid(dev):
    t = make_tree(dev, np.array([10, 20], np.uint64), np.array([1, 2], np.uint64))
    ref = oracle.MapOracle(); ref.load(np.array([10, 20], np.uint64), np.array([1, 2], np.uint64))
    run_and_compare(t, ref, np.array([3, 0], np.uint8), np.array([10, 10], np.uint64),
                    np.array([NF, 0], np.uint64), dev)


def test_host_buffer_path(dev):
    w = W.Workload(2, tree=1 << 14, batch=1 << 12)
    t = make_tree(dev, w.keys, w.vals, max_batch=1 << 12)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    ops, keys, vals = w.batch_arrays(0)
    res = torch.empty(ops.size, dtype=torch.uint64).pin_memory()
    tk = t.submit_host(torch.from_numpy(ops).pin_memory(), torch.from_numpy(keys).pin_memory(),
                       torch.from_numpy(vals).pin_memory(), res)
    t.results(tk)
    assert np.array_equal(res.numpy(), ref.apply(ops, keys, vals))


@pytest.mark.parametrize("pinned", [True, False])
def test_host_buffer_pipeline(dev, pinned):
    """Several host-path batches in flight (double-buffered staging, D2H on its
    own stream); pinned values are read zero-copy by the distribution kernel,
    pageable ones are copied."""
    w = W.Workload(4, tree=1 << 14, batch=1 << 12)
    t = make_tree(dev, w.keys, w.vals, max_batch=1 << 12, max_keys=1 << 17)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    pend = []
    for b in range(5):
        ops, keys, vals = w.batch_arrays(b)
        mk = (lambda a: torch.from_numpy(a).pin_memory()) if pinned else (lambda a: torch.from_numpy(a.copy()))
        res = torch.empty(ops.size, dtype=torch.uint64)
        if pinned:
            res = res.pin_memory()
        args = (mk(ops), mk(keys), mk(vals))
        pend.append((t.submit_host(*args, res), res, args, ref.apply(ops, keys, vals)))
    for tk, res, _, want in pend:
        t.results(tk)
        assert np.array_equal(res.numpy(), want)
    assert t.check_invariants()[0] == 0


def test_subbatch_splitting_invariance(dev):
    rng = np.random.default_rng(12)
    keys, vals = _rand_keys(rng, 2000, hi=1 << 16)
    n = 1 << 14
    ops = rng.integers(0, 4, n).astype(np.uint8)
    ks = rng.integers(1, 1 << 16, n, dtype=np.uint64)
    vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
    a = make_tree(dev, keys, vals, max_batch=n)
    ra, _ = a.apply(T(ops, dev), T(ks, dev), T(vs, dev))
    b = make_tree(dev, keys, vals, max_batch=n)
    parts = []
    for lo, hi in [(0, 100), (100, 5000), (5000, 5001), (5001, n)]:
        r, _ = b.apply(T(ops[lo:hi], dev), T(ks[lo:hi], dev), T(vs[lo:hi], dev))
        parts.append(r.cpu().numpy())
    assert np.array_equal(ra.cpu().numpy(), np.concatenate(parts))
    for x, y in zip(a.scan(), b.scan()):
        assert np.array_equal(x.cpu().numpy(), y.cpu().numpy())


def test_route_partition_unpermute(dev):
    rng = np.random.default_rng(21)
    n = 50000
    P = 8
    ks = rng.integers(1, 1 << 62, n, dtype=np.uint64)
    ops = rng.integers(0, 4, n).astype(np.uint8)
    vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
    sp = np.sort(rng.integers(1, 1 << 62, P - 1, dtype=np.uint64))
    t = make_tree(dev, np.empty(0, np.uint64), np.empty(0, np.uint64), max_batch=n)
    sops, skeys, svals, perm, counts = t.route_partition(T(ops, dev), T(ks, dev), T(vs, dev), T(sp, dev), P)
    dest = np.searchsorted(sp, ks, side="right")
    order = np.argsort(dest, kind="stable")
    assert np.array_equal(counts.cpu().numpy(), np.bincount(dest, minlength=P))
    assert np.array_equal(perm.cpu().numpy(), order)
    assert np.array_equal(skeys.cpu().numpy(), ks[order])
    assert np.array_equal(svals.cpu().numpy(), vs[order])
    assert np.array_equal(sops.cpu().numpy(), ops[order])
    back = t.route_unpermute(skeys, perm)
    assert np.array_equal(back.cpu().numpy(), ks)


def test_prepare_batch_then_submit(dev):
    """eirene_prepare_batch captures the graph without touching the tree; the
    batches that follow replay it and stay bit-exact."""
    rng = np.random.default_rng(77)
    keys, vals = _rand_keys(rng, 5000)
    t = make_tree(dev, keys, vals)
    t.prepare(4096)
    t.prepare(4096, ranges=True)
    k, v = t.scan()
    assert np.array_equal(k.cpu().numpy(), keys) and np.array_equal(v.cpu().numpy(), vals)
    ref = oracle.MapOracle()
    ref.load(keys, vals)
    for b in range(3):
        ops = rng.integers(0, 4, 4096).astype(np.uint8)
        ks = np.where(rng.random(4096) < 0.5, keys[rng.integers(0, keys.size, 4096)],
                      rng.integers(1, 1 << 40, 4096, dtype=np.uint64))
        vs = rng.integers(0, 1 << 62, 4096, dtype=np.uint64)
        run_and_compare(t, ref, ops, ks, vs, dev)


@pytest.mark.parametrize("zipf", [False, True])
def test_large_batch_two_kernel_sort(dev, zipf):
    """A batch above 2^22 requests (ragged size) takes the two-kernel bucket sort
    with 16384 bins (bsort.cu); with Zipf keys several groups are oversized."""
    from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W
    n = (1 << 22) + 4097
    w = W.Workload(3 if zipf else 2, tree=1 << 20, batch=n)
    t = make_tree(dev, w.keys, w.vals, max_keys=1 << 22, max_batch=n)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    for b in range(2):
        ops, keys, vals = w.batch_arrays(b)
        run_and_compare(t, ref, ops, keys, vals, dev, check_scan=(b == 1))
    t.close()


def test_narrow_shard_key_range(dev):
    """A shard owning a 2^40-wide slice of the key space: bins are taken over
    [key_lo, key_hi), not over the top bits of the key (bin_of)."""
    lo = 1 << 60
    rng = np.random.default_rng(77)
    keys = np.unique(rng.integers(lo, lo + (1 << 40), 50000, dtype=np.uint64))
    vals = rng.integers(0, 1 << 62, keys.size, dtype=np.uint64)
    t = make_tree(dev, keys, vals, max_batch=1 << 17, key_lo=lo, key_hi=lo + (1 << 40))
    ref = oracle.MapOracle(); ref.load(keys, vals)
    n = 1 << 17
    for b in range(2):
        ops = rng.integers(0, 4, n).astype(np.uint8)
        ks = np.where(rng.random(n) < 0.7, rng.choice(keys, n),
                      rng.integers(lo, lo + (1 << 40), n, dtype=np.uint64)).astype(np.uint64)
        vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
        run_and_compare(t, ref, ops, ks, vs, dev)
    assert t.check_invariants()[0] == 0
    t.close()


def test_edge_batches(dev):
    """Degenerate batches: a single request, extreme valid keys (0 and UINT64_MAX - 1)
    and values (UINT64_MAX - 1), queries / deletes on an empty tree, a batch of exactly
    max_batch requests, all-delete batches that empty the tree and a refill."""
    rng = np.random.default_rng(11)
    t = make_tree(dev, np.empty(0, np.uint64), np.empty(0, np.uint64), max_keys=1 << 14, max_batch=4096)
    ref = oracle.MapOracle()
    top = np.uint64(0xFFFFFFFFFFFFFFFE)
    # empty tree: queries and deletes of absent keys
    run_and_compare(t, ref, np.array([0, 3, 0], np.uint8), np.array([0, 5, top], np.uint64),
                    np.zeros(3, np.uint64), dev)
    # one request at a time, extreme keys and values
    for op, k, v in [(2, 0, top), (2, top, 1), (0, 0, 0), (1, top, top), (0, top, 0), (3, 0, 0), (0, 0, 0)]:
        run_and_compare(t, ref, np.array([op], np.uint8), np.array([k], np.uint64), np.array([v], np.uint64), dev)
    # exactly max_batch requests over a small key set (long segments, splits from a 1-key tree)
    n = 4096
    ops = rng.integers(0, 4, n).astype(np.uint8)
    ks = rng.integers(0, 600, n, dtype=np.uint64) * np.uint64(0x9E3779B97F4A7C15 >> 4)
    vs = rng.integers(0, 1 << 63, n, dtype=np.uint64)
    run_and_compare(t, ref, ops, ks, vs, dev)
    # delete everything, then query it all, then refill
    live, _ = ref.scan()
    d = np.resize(live, n) if live.size else np.zeros(n, np.uint64)
    run_and_compare(t, ref, np.full(n, 3, np.uint8), d, np.zeros(n, np.uint64), dev)
    run_and_compare(t, ref, np.zeros(n, np.uint8), d, np.zeros(n, np.uint64), dev)
    assert ref.size() == 0
    run_and_compare(t, ref, np.full(n, 2, np.uint8), d, vs, dev)
    assert t.check_invariants()[0] == 0
    t.close()


def test_efull_rejects_batch_untouched(dev):
    """Pool headroom: a batch whose worst case (every issued write
    an insert that splits) exceeds the leaf pool is rejected with EFULL before any
    kernel modifies the tree; the tree then still serves batches that fit."""
    from paper_conf_ppopp_zhangz0lzl23_b200._ffi import EIRENE_EFULL
    rng = np.random.default_rng(21)
    nb = 4096
    # leaf_cap = max_keys / 8 + 2 * max_batch + 1024 = 9728 leaves (api.cu); one key per leaf
    keys = np.arange(1, 9001, dtype=np.uint64) * np.uint64(1 << 20)
    vals = rng.integers(0, 1 << 62, keys.size, dtype=np.uint64)
    t = make_tree(dev, keys, vals, max_keys=4096, max_batch=nb, fill=1.0 / 16)
    assert t.info()["leaves"] == 9000
    ref = oracle.MapOracle(); ref.load(keys, vals)
    ops = np.full(nb, 2, np.uint8)
    ks = keys[:nb] + np.uint64(1)           # 4096 distinct fresh keys: 9000 + 4096 > 9728
    vs = rng.integers(0, 1 << 62, nb, dtype=np.uint64)
    res = torch.empty(nb, dtype=torch.uint64, device=dev)
    st = t.results(t.submit(T(ops, dev), T(ks, dev), T(vs, dev), res), raise_on_error=False)
    assert st["rc"] == EIRENE_EFULL and st["status"] == EIRENE_EFULL
    k, v = t.scan()
    assert np.array_equal(k.cpu().numpy(), keys) and np.array_equal(v.cpu().numpy(), vals)
    assert t.check_invariants() == (0, keys.size)
    # a batch within the headroom goes through: 500 fresh inserts (the bound counts every
    # issued write as a potential new leaf: 9000 + 500 <= 9728), the rest queries
    ops2 = np.where(np.arange(nb) < 500, 2, 0).astype(np.uint8)
    ks2 = np.where(np.arange(nb) < 500, ks, keys[rng.integers(0, keys.size, nb)]).astype(np.uint64)
    run_and_compare(t, ref, ops2, ks2, vs, dev)
    t.close()


@pytest.mark.parametrize("zipf", [False, True])
def test_two_kernel_sort_size_band(dev, zipf):
    """Batches above the fused distribution kernel's capacity (one resident
    wave, ~1.2M requests) but at most 2^22 take the two-kernel path with its
    own 16384-bin buffers (bsort_fused decides for the launcher, the group
    count and the buffers alike) -- the per-shard batch of cfg5 at N = 4 / 8."""
    from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W
    n = (1 << 21) + 123
    w = W.Workload(3 if zipf else 2, tree=1 << 20, batch=n)
    t = make_tree(dev, w.keys, w.vals, max_keys=1 << 22, max_batch=n)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    for b in range(2):
        ops, keys, vals = w.batch_arrays(b)
        run_and_compare(t, ref, ops, keys, vals, dev, check_scan=(b == 1))
    t.close()


@pytest.mark.parametrize("n", [1_100_000, (1 << 21) + 77])
def test_two_phase_group_stage(dev, n):
    """More groups than one resident wave (2 per SM): the group stage runs as
    two kernels -- sort + aggregates, then look-back + emit (group.cu) -- on
    Zipf keys with every op kind, so small, L2-sorted and SPLIT (hot-key
    bitmap) groups all cross the phase boundary; n = 1.1M stays on the fused
    distribution kernel, 2^21 + 77 takes the two-kernel one."""
    from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W
    w = W.Workload(3, tree=1 << 20, batch=n, fracs={0: 0.4, 1: 0.2, 2: 0.3, 3: 0.1})
    t = make_tree(dev, w.keys, w.vals, max_keys=1 << 22, max_batch=n)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    for b in range(2):
        ops, keys, vals = w.batch_arrays(b)
        run_and_compare(t, ref, ops, keys, vals, dev, check_scan=(b == 1))
    assert t.check_invariants()[0] == 0
    t.close()


def test_structural_counts_and_device_time(dev):
    """nins / ndelp (the structural writes the update kernel is left with; value
    overwrites are applied in place by the query kernel) equal their definition
    on the oracle's pre-batch state, and the device batch time is recorded."""
    rng = np.random.default_rng(5)
    keys, vals = _rand_keys(rng, 20000)
    t = make_tree(dev, keys, vals, max_batch=1 << 15)
    ref = oracle.MapOracle(); ref.load(keys, vals)
    for b in range(3):
        n = 1 << 15
        ops = rng.integers(0, 4, n).astype(np.uint8)
        if b == 2:
            ops[ops >= 2] = 1               # overwrites only: the update kernel has nothing left
        ks = np.where(rng.random(n) < 0.6, keys[rng.integers(0, keys.size, n)],
                      rng.integers(1, 1 << 40, n, dtype=np.uint64)).astype(np.uint64)
        vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
        pre_k, _ = ref.scan()
        if b == 2:   # every write on a live key
            ks[ops == 1] = pre_k[rng.integers(0, pre_k.size, int(np.sum(ops == 1)))]
        # issued write per key = its last write; structural iff insert of absent / delete of present
        last = {}
        for o, k in zip(ops, ks):
            if o != 0:
                last[int(k)] = int(o)
        present = set(int(x) for x in pre_k)
        want_ins = sum(1 for k, o in last.items() if o != 3 and k not in present)
        want_delp = sum(1 for k, o in last.items() if o == 3 and k in present)
        st = run_and_compare(t, ref, ops, ks, vs, dev)
        assert (st["nins"], st["ndelp"]) == (want_ins, want_delp)
        if b == 2:
            assert want_ins == 0 and want_delp == 0
        assert 0 < st["device_ns"] < 10**9
    t.close()


@pytest.mark.parametrize("cfg", [2, 3])
def test_pipelined_batches_in_flight(dev, cfg):
    """EIRENE_F_PIPELINE (§8(f) NEXT(3)): the front (sort, combine, partition) of
    batch b+1 overlaps the back (query, update, RESULT_CAL) of batch b.  Many
    batches are submitted before any result is read; every result and the final
    state must equal the oracle's (backs in submission order), and a
    non-pipelined batch and a scan afterwards must see every pipelined one."""
    rng = np.random.default_rng(40 + cfg)
    w = W.Workload(cfg, tree=1 << 16, batch=1 << 14,
                   fracs={W.QUERY: 0.5, W.UPDATE: 0.25, W.INSERT: 0.2, W.DELETE: 0.05})
    t = make_tree(dev, w.keys, w.vals, max_keys=1 << 18, max_batch=1 << 14, pipeline=True)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    nb = 9
    host = [w.batch_arrays(b) for b in range(nb)]
    outs, tks = [], []
    for b in range(nb):
        n = (1 << 14) - int(rng.integers(0, 3000))   # ragged sizes: several graph buckets
        o, k, v = (T(a[:n], dev) for a in host[b])
        res = torch.empty(n, dtype=torch.uint64, device=dev)
        tks.append(t.submit(o, k, v, res))
        outs.append((res, n, (o, k, v)))
    for b in range(nb):
        st = t.results(tks[b])
        res, n, _ = outs[b]
        want = ref.apply(host[b][0][:n], host[b][1][:n], host[b][2][:n])
        got = res.cpu().numpy()
        assert np.array_equal(got, want), f"batch {b}: {int(np.sum(got != want))} differ"
    k, v = t.scan()
    rk, rv = ref.scan()
    assert np.array_equal(k.cpu().numpy(), rk) and np.array_equal(v.cpu().numpy(), rv)
    # the host-buffer path on a pipelined handle
    o, k_, v_ = w.batch_arrays(50)
    pin = [torch.from_numpy(a).pin_memory() for a in (o, k_, v_)]
    hres = torch.empty(o.size, dtype=torch.uint64).pin_memory()
    t.results(t.submit_host(*pin, hres))
    assert np.array_equal(hres.numpy(), ref.apply(o, k_, v_))
    assert t.check_invariants() == (0, ref.size())
    t.close()
