"""GPU parity for range queries R(l, u) (§4.1.2,
P:848-1042): the CUDA path through eirene_submit_batch_range vs the CPU
oracle's definition engine (MapOracle.apply_range), bit-exact on every
per-request result, every range row and the final scan.  Run with -m gpu."""
import json
import os

import numpy as np
import pytest
import torch

import oracle
from oracle import RANGE
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


def run_range(t, ref, ops, keys, vals, cap, dev, check_scan=True):
    res, rk, rv, st = t.apply_range(T(ops, dev), T(keys, dev), T(vals, dev), cap)
    want, wk, wv = ref.apply_range(ops, keys, vals, cap)
    got = res.cpu().numpy()
    bad = np.nonzero(got != want)[0]
    assert bad.size == 0, (f"{bad.size} of {len(ops)} results differ; first at {bad[:5]}: "
                           f"got {got[bad[:5]]}, want {want[bad[:5]]}, ops {ops[bad[:5]]}")
    r = np.nonzero(ops == RANGE)[0]
    gk, gv = rk.cpu().numpy(), rv.cpu().numpy()
    for name, g, w in (("keys", gk, wk), ("vals", gv, wv)):
        for i in r:
            c = int(want[i])
            assert np.array_equal(g[i, :c], w[i, :c]), f"range row {i} {name}: got {g[i, :c]}, want {w[i, :c]}"
    assert st["ranges"] == r.size
    if check_scan:
        k, v = t.scan()
        sk, sv = ref.scan()
        assert np.array_equal(k.cpu().numpy(), sk) and np.array_equal(v.cpu().numpy(), sv), "scan differs"
    return st


def _fig(golden_dir, name):
    with open(os.path.join(golden_dir, name)) as f:
        g = json.load(f)
    val = g["values"]
    OPC = {"Q": 0, "U": 1, "I": 2, "D": 3, "R": RANGE}
    pk = np.array([k for k, _ in g["pre_batch"]], dtype=np.uint64)
    pv = np.array([val[v] for _, v in g["pre_batch"]], dtype=np.uint64)
    reqs = sorted(g["requests"], key=lambda r: r["ts"])
    ops = np.array([OPC[r["op"]] for r in reqs], np.uint8)
    keys = np.array([r["lo"] if r["op"] == "R" else r["key"] for r in reqs], np.uint64)
    vals = np.array([r["hi"] if r["op"] == "R" else val.get(r.get("val"), 0) for r in reqs], np.uint64)
    return g, val, pk, pv, ops, keys, vals, {r["ts"]: i for i, r in enumerate(reqs)}


@pytest.mark.parametrize("fig", ["fig4.json", "fig5.json"])
def test_paper_range_examples(dev, golden_dir, fig):
    g, val, pk, pv, ops, keys, vals, tsi = _fig(golden_dir, fig)
    t = make_tree(dev, pk, pv)
    res, rk, rv, st = t.apply_range(T(ops, dev), T(keys, dev), T(vals, dev), 8)
    res, rk, rv = res.cpu().numpy(), rk.cpu().numpy(), rv.cpu().numpy()
    for part in ("expected_range_paper", "expected_range_reading"):
        for ts, kv in g.get(part, {}).items():
            if ts.startswith("_"):
                continue
            i = tsi[int(ts)]
            got = {int(rk[i, j]): int(rv[i, j]) for j in range(int(res[i]))}
            assert got == {int(k): val[v] for k, v in kv.items()} or part == "expected_range_paper" and all(
                got.get(int(k)) == val[v] for k, v in kv.items())
    for ts, v in g.get("expected_results_paper", {}).items():
        if not ts.startswith("_"):
            assert int(res[tsi[int(ts)]]) == val[v]
    if "artificial_queries" in g:
        assert st["artificial"] == g["artificial_queries"]["count"]
    k, v = t.scan()
    assert [(int(a), int(b)) for a, b in zip(k.cpu().numpy(), v.cpu().numpy())] == \
        [(kk, val[vv]) for kk, vv in g["final_state"]]


@pytest.mark.parametrize("cap", [1, 3, 16, 100])
def test_range_only_batches(dev, cap):
    """No writes: every range reads the bulk-loaded tree, crossing leaves;
    empty (l > u), unbounded (u = UINT64_MAX), below-all and above-all ranges."""
    rng = np.random.default_rng(cap)
    keys = np.unique(rng.integers(1, 1 << 40, 50000, dtype=np.uint64))
    vals = rng.integers(0, 1 << 62, keys.size, dtype=np.uint64)
    t = make_tree(dev, keys, vals, fill=0.8)
    ref = oracle.MapOracle()
    ref.load(keys, vals)
    n = 20000
    ops = np.full(n, RANGE, np.uint8)
    j = rng.integers(0, keys.size, n)
    lo = keys[j] - rng.integers(0, 2, n).astype(np.uint64)
    span = rng.integers(0, 200, n)
    hi = keys[np.minimum(j + span, keys.size - 1)] + rng.integers(0, 2, n).astype(np.uint64)
    lo[:50] = hi[:50] + np.uint64(1)                 # empty
    hi[50:100] = NF                                  # unbounded above
    lo[100:110] = 0
    lo[110:120] = np.uint64(1 << 41)                 # above every key
    lo[120:130] = NF
    hi[120:130] = NF
    run_range(t, ref, ops, lo, hi, cap, dev)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_mixed_conflict_heavy(dev, seed):
    """All five request types on a small key space (many keys per segment,
    ranges overlapping written, inserted and deleted keys); several batches."""
    rng = np.random.default_rng(40 + seed)
    keys = np.unique(rng.integers(0, 3000, 1500, dtype=np.uint64))
    vals = rng.integers(0, 1 << 62, keys.size, dtype=np.uint64)
    t = make_tree(dev, keys, vals, max_keys=1 << 14)
    ref = oracle.MapOracle()
    ref.load(keys, vals)
    for b in range(6):
        n = int(rng.integers(1000, 20000))
        ops = rng.choice(np.arange(5, dtype=np.uint8), n, p=[0.3, 0.2, 0.15, 0.15, 0.2])
        ks = rng.integers(0, 3000, n, dtype=np.uint64)
        vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
        r = ops == RANGE
        vs[r] = ks[r] + rng.integers(0, 60, int(r.sum()), dtype=np.uint64)
        run_range(t, ref, ops, ks, vs, int(rng.integers(1, 48)), dev)
    rc, nk = t.check_invariants()
    assert rc == 0 and nk == ref.size()


def test_hot_key_long_segment(dev):
    """One key with ~30K requests (a long, oversized segment) and ranges at
    many timestamps over it: the artificial query's binary search over the
    segment must find the nearest earlier write for every range."""
    rng = np.random.default_rng(7)
    keys = np.arange(100, 200, dtype=np.uint64) * np.uint64(2)
    vals = keys + np.uint64(1)
    t = make_tree(dev, keys, vals)
    ref = oracle.MapOracle()
    ref.load(keys, vals)
    n = 60000
    ops = rng.choice(np.arange(5, dtype=np.uint8), n, p=[0.3, 0.3, 0.05, 0.1, 0.25])
    ks = np.full(n, 300, np.uint64)
    ks[rng.random(n) < 0.3] = np.uint64(302)
    vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
    r = ops == RANGE
    vs[r] = np.uint64(310)
    ks[r] = np.uint64(290)
    run_range(t, ref, ops, ks, vs, 16, dev)


def test_ranges_over_emptied_leaves(dev):
    """Delete whole runs of keys (leaves stay linked but empty, no
    rebalancing), then range over them: the walk crosses empty leaves."""
    keys = np.arange(1, 20001, dtype=np.uint64) * np.uint64(4)
    vals = keys * np.uint64(3)
    t = make_tree(dev, keys, vals)
    ref = oracle.MapOracle()
    ref.load(keys, vals)
    dele = keys[(keys > 4000) & (keys < 60000)]
    ops = np.full(dele.size, W.DELETE, np.uint8)
    z = np.zeros(dele.size, np.uint64)
    res, _, _, _ = t.apply_range(T(ops, dev), T(dele, dev), T(z, dev), 4)
    ref.apply(ops, dele, z)
    n = 4000
    rng = np.random.default_rng(3)
    ops = np.full(n, RANGE, np.uint8)
    lo = rng.integers(0, 90000, n, dtype=np.uint64)
    hi = lo + rng.integers(0, 70000, n, dtype=np.uint64)
    run_range(t, ref, ops, lo, hi, 24, dev)


def test_workload_ranges_with_writes(dev):
    """The generator's range requests (length-8 ranges over loaded keys) mixed
    with cfg2-style queries and updates and with inserts/deletes, on a 2^18-key
    tree, at a batch large enough for many groups."""
    w = W.Workload(2, tree=1 << 18, batch=1 << 17,
                   fracs={W.QUERY: 0.4, W.UPDATE: 0.2, W.INSERT: 0.1, W.DELETE: 0.05, W.RANGE: 0.25})
    t = make_tree(dev, w.keys, w.vals, max_keys=1 << 20, max_batch=1 << 17)
    ref = oracle.MapOracle()
    ref.load(w.keys, w.vals)
    for b in range(3):
        ops, keys, vals = w.batch_arrays(b)
        run_range(t, ref, ops, keys, vals, 8, dev, check_scan=(b == 2))


def test_range_op_rejected_without_range_outputs(dev):
    from paper_conf_ppopp_zhangz0lzl23_b200._ffi import EireneError
    keys = np.arange(10, 100, dtype=np.uint64)
    t = make_tree(dev, keys, keys)
    ops = np.array([W.UPDATE, RANGE], np.uint8)
    ks = np.array([10, 10], np.uint64)
    vs = np.array([5, 50], np.uint64)
    with pytest.raises(EireneError):
        t.apply(T(ops, dev), T(ks, dev), T(vs, dev))
    k, v = t.scan()
    assert np.array_equal(v.cpu().numpy(), keys)      # tree untouched
    # the same batch through the range entry point is valid
    ref = oracle.MapOracle()
    ref.load(keys, keys)
    run_range(t, ref, ops, ks, vs, 4, dev)


def test_single_range_and_point_free_batch(dev):
    keys = np.arange(0, 64, dtype=np.uint64) * np.uint64(10)
    t = make_tree(dev, keys, keys + np.uint64(7))
    ref = oracle.MapOracle()
    ref.load(keys, keys + np.uint64(7))
    run_range(t, ref, np.array([RANGE], np.uint8), np.array([95], np.uint64), np.array([400], np.uint64), 64, dev)
    run_range(t, ref, np.array([RANGE] * 3, np.uint8), np.array([0, 630, 5], np.uint64),
              np.array([0, 10 ** 6, 4], np.uint64), 2, dev)
