"""Pins for the CPU oracle (runs without a GPU).

Each test pins the oracle to something other than itself:
the paper's Fig.3 worked example (tests/golden/fig3.json), special
cases that reduce to library routines (numpy searchsorted / union), closed
forms of the per-key dependence rule, metamorphic invariants
(sub-batch splitting, commutativity of distinct keys) and B+tree invariants.
"""
import itertools
import json
import os

import numpy as np
import pytest

import oracle
from oracle import NOT_FOUND, BTreeOracle, MapOracle, combine_apply
from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W

OPC = {"Q": 0, "U": 1, "I": 2, "D": 3}
NF = int(NOT_FOUND)


def _fig3(golden_dir):
    with open(os.path.join(golden_dir, "fig3.json")) as f:
        g = json.load(f)
    val = g["values"]
    pre_k = np.array([k for k, _ in g["pre_batch"]], dtype=np.uint64)
    pre_v = np.array([val[v] for _, v in g["pre_batch"]], dtype=np.uint64)
    reqs = sorted(g["requests"], key=lambda r: r["ts"])
    ops = np.array([OPC[r["op"]] for r in reqs], dtype=np.uint8)
    keys = np.array([r["key"] for r in reqs], dtype=np.uint64)
    vals = np.array([val[r["val"]] if "val" in r else 0 for r in reqs], dtype=np.uint64)
    exp = {}
    for part in ("expected_results_paper", "expected_results_reading1"):
        for ts, v in g[part].items():
            if not ts.startswith("_"):
                exp[int(ts)] = val[v]
    return g, val, pre_k, pre_v, ops, keys, vals, exp


def _check_fig3_results(res, exp):
    # timestamps in the fixture are 1-based (T1..T8); batch index = ts - 1
    for ts, v in exp.items():
        assert int(res[ts - 1]) == v, f"T{ts}: got {int(res[ts - 1])}, want {v}"


def test_fig3_map(golden_dir):
    g, val, pk, pv, ops, keys, vals, exp = _fig3(golden_dir)
    m = MapOracle()
    m.load(pk, pv)
    _check_fig3_results(m.apply(ops, keys, vals), exp)
    k, v = m.scan()
    assert [(int(a), int(b)) for a, b in zip(k, v)] == [(kk, val[vv]) for kk, vv in g["final_state"]]


@pytest.mark.parametrize("fanout", [3, 4, 16])
def test_fig3_btree(golden_dir, fanout):
    g, val, pk, pv, ops, keys, vals, exp = _fig3(golden_dir)
    t = BTreeOracle(fanout)
    t.load(pk, pv)
    _check_fig3_results(t.apply(ops, keys, vals), exp)
    k, v = t.scan()
    assert [(int(a), int(b)) for a, b in zip(k, v)] == [(kk, val[vv]) for kk, vv in g["final_state"]]
    assert t.check() == 0


def test_fig3_combining(golden_dir):
    g, val, pk, pv, ops, keys, vals, exp = _fig3(golden_dir)
    m = MapOracle()
    m.load(pk, pv)
    out = combine_apply(m, ops, keys, vals)
    _check_fig3_results(out["results"], exp)
    # sorted order (Fig.3(b)), 1-based timestamps
    assert [int(t) + 1 for t in out["sorted_ts"]] == g["sorted_ts"]
    assert out["n_issued"] == len(g["issued"])
    for s, iss in enumerate(g["issued"]):
        assert int(out["issued_key"][s]) == iss["key"]
        assert int(out["issued_op"][s]) == OPC[iss["op"]]
        if "val" in iss:
            assert int(out["issued_val"][s]) == val[iss["val"]]
    assert out["n_issued_w"] == 2
    k, v = m.scan()
    assert [(int(a), int(b)) for a, b in zip(k, v)] == [(kk, val[vv]) for kk, vv in g["final_state"]]


def _rand_tree(rng, n, lo=0, hi=1 << 40):
    keys = np.unique(rng.integers(lo, hi, size=n * 2, dtype=np.uint64))[:n]
    vals = rng.integers(0, 1 << 62, size=keys.size, dtype=np.uint64)
    return keys, vals


@pytest.mark.parametrize("engine", ["map", "bt"])
def test_query_only_is_lower_bound(engine):
    """Special case: a query-only batch == std::lower_bound (numpy searchsorted)
    over the loaded sorted arrays; NOT_FOUND on a miss."""
    rng = np.random.default_rng(1)
    keys, vals = _rand_tree(rng, 5000)
    e = MapOracle() if engine == "map" else BTreeOracle(16)
    e.load(keys, vals)
    q = np.concatenate([keys[rng.integers(0, keys.size, 3000)],
                        rng.integers(0, 1 << 40, 3000, dtype=np.uint64)])
    rng.shuffle(q)
    res = e.apply(np.zeros(q.size, np.uint8), q, np.zeros(q.size, np.uint64))
    pos = np.searchsorted(keys, q)
    hit = (pos < keys.size) & (keys[np.minimum(pos, keys.size - 1)] == q)
    want = np.where(hit, vals[np.minimum(pos, keys.size - 1)], NOT_FOUND)
    assert np.array_equal(res, want)


@pytest.mark.parametrize("engine", ["map", "bt"])
def test_distinct_upserts_are_merge_with_overwrite(engine):
    """Special case: distinct-key upserts == union of the key sets with the new
    values overwriting; each write returns the pre-batch value."""
    rng = np.random.default_rng(2)
    keys, vals = _rand_tree(rng, 4000)
    e = MapOracle() if engine == "map" else BTreeOracle(5)
    e.load(keys, vals)
    wk = np.unique(np.concatenate([keys[rng.integers(0, keys.size, 1500)],
                                   rng.integers(0, 1 << 40, 1500, dtype=np.uint64)]))
    rng.shuffle(wk)
    wv = rng.integers(0, 1 << 62, wk.size, dtype=np.uint64)
    ops = rng.choice(np.array([1, 2], np.uint8), wk.size)
    res = e.apply(ops, wk, wv)
    pos = np.searchsorted(keys, wk)
    hit = (pos < keys.size) & (keys[np.minimum(pos, keys.size - 1)] == wk)
    assert np.array_equal(res, np.where(hit, vals[np.minimum(pos, keys.size - 1)], NOT_FOUND))
    allk = np.union1d(keys, wk)
    allv = np.empty(allk.size, np.uint64)
    allv[np.searchsorted(allk, keys)] = vals
    allv[np.searchsorted(allk, wk)] = wv
    k, v = e.scan()
    assert np.array_equal(k, allk) and np.array_equal(v, allv)
    if engine == "bt":
        assert e.check() == 0


def _nearest_write_closed_form(init, ops, keys, vals):
    """Per-key closed form of the dependence rule: the
    result of request i is the value of the NEAREST earlier write on its key
    (NOT_FOUND if that write is a delete), else the pre-batch value."""
    n = len(ops)
    res = []
    for i in range(n):
        r = init.get(int(keys[i]), NF)
        for j in range(i - 1, -1, -1):
            if keys[j] == keys[i] and ops[j] != 0:
                r = NF if ops[j] == 3 else int(vals[j])
                break
        res.append(r)
    return res


def test_exhaustive_tiny_alphabet():
    """Brute force: every request sequence of length <= 4 over 2 keys x
    {Q, U(a), U(b), I(a), D} (10 choices per position), from each of the 4
    initial presence states, against the closed form and final state."""
    alphabet = [(op, k, v) for k in (10, 20) for (op, v) in ((0, 0), (1, 7), (1, 8), (2, 7), (3, 0))]
    inits = [{}, {10: 1}, {20: 2}, {10: 1, 20: 2}]
    count = 0
    for init in inits:
        ik = np.array(sorted(init), dtype=np.uint64)
        iv = np.array([init[k] for k in sorted(init)], dtype=np.uint64)
        for L in range(1, 5):
            for seq in itertools.product(alphabet, repeat=L):
                ops = np.array([s[0] for s in seq], np.uint8)
                keys = np.array([s[1] for s in seq], np.uint64)
                vals = np.array([s[2] for s in seq], np.uint64)
                want = _nearest_write_closed_form(init, ops, keys, vals)
                m = MapOracle(); m.load(ik, iv)
                assert [int(x) for x in m.apply(ops, keys, vals)] == want
                c = MapOracle(); c.load(ik, iv)
                out = combine_apply(c, ops, keys, vals)
                assert [int(x) for x in out["results"]] == want
                assert np.array_equal(m.scan()[0], c.scan()[0]) and np.array_equal(m.scan()[1], c.scan()[1])
                # final state closed form: the last write per key decides
                fin = dict(init)
                for o, k, v in seq:
                    if o in (1, 2):
                        fin[k] = v
                    elif o == 3:
                        fin.pop(k, None)
                fk, fv = m.scan()
                assert {int(a): int(b) for a, b in zip(fk, fv)} == fin
                count += 1
    assert count == 4 * sum(10 ** L for L in range(1, 5))


@pytest.mark.parametrize("fanout", [3, 4, 5, 16])
def test_btree_vs_map_random_streams(fanout):
    rng = np.random.default_rng(100 + fanout)
    keys, vals = _rand_tree(rng, 300, 0, 2000)
    m, t = MapOracle(), BTreeOracle(fanout)
    m.load(keys, vals); t.load(keys, vals)
    assert t.check() == 0
    for b in range(60):
        n = int(rng.integers(1, 60))
        ops = rng.integers(0, 4, n).astype(np.uint8)
        ks = rng.integers(0, 2000, n, dtype=np.uint64)
        vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
        assert np.array_equal(m.apply(ops, ks, vs), t.apply(ops, ks, vs))
        assert t.check() == 0, f"invariant {t.check()} after batch {b}"
        assert t.size() == m.size()
    for a, b in zip(m.scan(), t.scan()):
        assert np.array_equal(a, b)
    # drain to empty: deletes everywhere exercise borrow/merge down to the root
    live = m.scan()[0]
    d = live[rng.permutation(live.size)]
    t.apply(np.full(d.size, 3, np.uint8), d, np.zeros(d.size, np.uint64))
    assert t.check() == 0 and t.size() == 0 and t.height() == 1


def test_btree_single_ops_keep_invariants():
    """Invariants after EVERY operation on a small-fanout tree."""
    rng = np.random.default_rng(7)
    m, t = MapOracle(), BTreeOracle(3)
    for i in range(1500):
        op = np.array([rng.integers(0, 4)], np.uint8)
        k = np.array([rng.integers(0, 200)], np.uint64)
        v = np.array([rng.integers(0, 1000)], np.uint64)
        assert np.array_equal(m.apply(op, k, v), t.apply(op, k, v))
        assert t.check() == 0


@pytest.mark.parametrize("kind,code", [(1, 1), (2, 2), (5, 5), (6, 6)])
def test_btree_checker_detects_corruption(kind, code):
    keys = np.arange(0, 400, 2, dtype=np.uint64)
    t = BTreeOracle(4)
    t.load(keys, keys + 1)
    assert t.check() == 0
    assert t.corrupt(kind) == 0
    assert t.check() == code


# Codes 3 (unequal leaf depth), 4 (fill outside [ceil(F/2), F] below the root,
# both directions) and 7 (shape: #keys != #values) -- the "fill bounds, uniform
# leaf depth" invariants of the B+tree that north_star names.
@pytest.mark.parametrize("F", [3, 4, 5, 16])
@pytest.mark.parametrize("kind,code", [(4, 4), (7, 7), (8, 4)])
def test_btree_checker_detects_fill_shape(F, kind, code):
    rng = np.random.default_rng(100 + F)
    t = BTreeOracle(F)
    keys = rng.permutation(np.arange(0, 4000, 2, dtype=np.uint64))
    t.apply(np.full(keys.size, 2, np.uint8), keys, keys + 1)
    assert t.check() == 0 and t.height() >= 3
    assert t.corrupt(kind) == 0
    assert t.check() == code


@pytest.mark.parametrize("F", [3, 5, 16])
def test_btree_depth_corruption_needs_small_fanout(F):
    """A depth-only defect (a leaf pushed under a new 2-child inner node, every
    other invariant intact) exists only when 2 children and 2 half-full leaves
    are legal: F = 4.  Other fanouts: the hook refuses (F odd: no leaf splits into
    two legal leaves) or the new node breaks fill first (F = 16: code 4)."""
    t = BTreeOracle(F)
    keys = np.random.default_rng(F).permutation(np.arange(0, 4000, 2, dtype=np.uint64))
    t.apply(np.full(keys.size, 2, np.uint8), keys, keys + 1)
    rc = t.corrupt(3)
    if F in (3, 5):
        assert rc == -1 and t.check() == 0
    else:
        assert rc == 0 and t.check() == 4


def test_btree_checker_depth_only_violation_is_first_reported():
    """A tree whose ONLY defect is unequal leaf depth (fill, order, fences, chain
    and size all valid) must fail with 3, not pass: a checker that never tests
    depth would accept it."""
    t = BTreeOracle(4)
    keys = np.random.default_rng(3).permutation(np.arange(0, 2000, 2, dtype=np.uint64))
    t.apply(np.full(keys.size, 2, np.uint8), keys, keys + 1)
    n0 = t.size()
    assert t.corrupt(3) == 0
    assert t.size() == n0
    # every key is still found with its value, in order (the defect is structural only)
    assert np.array_equal(t.scan(0, 1 << 62)[0], np.sort(keys))
    assert t.check() == 3


def test_combining_vs_map_conflict_heavy():
    rng = np.random.default_rng(11)
    keys, vals = _rand_tree(rng, 200, 0, 400)
    m, c = MapOracle(), MapOracle()
    m.load(keys, vals); c.load(keys, vals)
    for b in range(30):
        n = int(rng.integers(1, 3000))
        ops = rng.integers(0, 4, n).astype(np.uint8)
        ks = rng.integers(0, 400, n, dtype=np.uint64)
        vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
        want = m.apply(ops, ks, vs)
        out = combine_apply(c, ops, ks, vs)
        assert np.array_equal(out["results"], want)
        # invariants: #issued = #distinct keys; issued op = last write else QUERY
        uk = np.unique(ks)
        assert out["n_issued"] == uk.size
        assert np.array_equal(out["issued_key"], uk)
        for s, k in enumerate(uk):
            idx = np.nonzero(ks == k)[0]
            wr = idx[ops[idx] != 0]
            if wr.size:
                assert out["issued_op"][s] == ops[wr[-1]]
            else:
                assert out["issued_op"][s] == 0
                assert len(set(int(x) for x in out["results"][idx])) == 1   # all-query: all equal
        assert out["n_issued_w"] == int(np.sum(out["issued_op"] != 0))
        # sorted_ts is the stable sort by key
        assert np.array_equal(out["sorted_ts"], np.argsort(ks, kind="stable").astype(np.uint32))
    for a, b in zip(m.scan(), c.scan()):
        assert np.array_equal(a, b)


def test_subbatch_splitting_invariance():
    """Metamorphic (SURVEY §8(c) reading 9): results are invariant under
    splitting a batch into consecutive sub-batches."""
    rng = np.random.default_rng(5)
    keys, vals = _rand_tree(rng, 500, 0, 1000)
    n = 4000
    ops = rng.integers(0, 4, n).astype(np.uint8)
    ks = rng.integers(0, 1000, n, dtype=np.uint64)
    vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
    a = MapOracle(); a.load(keys, vals)
    whole = combine_apply(a, ops, ks, vs)["results"]
    b = MapOracle(); b.load(keys, vals)
    cuts = np.sort(rng.choice(np.arange(1, n), 7, replace=False))
    parts = [combine_apply(b, o, k, v)["results"] for o, k, v in
             zip(np.split(ops, cuts), np.split(ks, cuts), np.split(vs, cuts))]
    assert np.array_equal(whole, np.concatenate(parts))
    for x, y in zip(a.scan(), b.scan()):
        assert np.array_equal(x, y)


def test_distinct_keys_commute():
    """Requests on different keys commute: permuting whole
    per-key subsequences (keeping each key's internal order) changes no result."""
    rng = np.random.default_rng(9)
    keys, vals = _rand_tree(rng, 100, 0, 300)
    n = 2000
    ops = rng.integers(0, 4, n).astype(np.uint8)
    ks = rng.integers(0, 300, n, dtype=np.uint64)
    vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
    a = MapOracle(); a.load(keys, vals)
    r1 = a.apply(ops, ks, vs)
    order = np.argsort(ks, kind="stable")          # group by key, keep per-key order
    b = MapOracle(); b.load(keys, vals)
    r2 = b.apply(ops[order], ks[order], vs[order])
    assert np.array_equal(r1[order], r2)


def test_invalid_requests_rejected():
    m = MapOracle()
    with pytest.raises(ValueError):
        m.apply(np.array([4], np.uint8), np.array([1], np.uint64), np.array([0], np.uint64))
    with pytest.raises(ValueError):
        m.apply(np.array([0], np.uint8), np.array([NF], np.uint64), np.array([0], np.uint64))
    with pytest.raises(ValueError):
        m.apply(np.array([1], np.uint8), np.array([1], np.uint64), np.array([NF], np.uint64))
    # a delete's value is ignored (even UINT64_MAX)
    m.apply(np.array([3], np.uint8), np.array([1], np.uint64), np.array([NF], np.uint64))


def test_workload_generator_shapes():
    w = W.Workload(2, tree=1 << 12, batch=1 << 12)
    assert w.keys.size == 1 << 12 and np.all(np.diff(w.keys.astype(np.float64)) >= 0)
    assert np.all(w.keys % 2 == 0)
    ops, keys, vals = w.batch_arrays(0)
    assert int(np.sum(ops == 0)) == round(0.95 * 4096) and int(np.sum(ops == 1)) == 4096 - round(0.95 * 4096)
    assert np.all(np.isin(keys, w.keys))
    o2, k2, v2 = W.Workload(2, tree=1 << 12, batch=1 << 12).batch_arrays(0)
    assert np.array_equal(ops, o2) and np.array_equal(keys, k2) and np.array_equal(vals, v2)
    w1 = W.Workload(1, tree=1 << 10, batch=1 << 10)
    o, k, v = w1.batch_arrays(0)
    assert np.all(k[o == 2] % 2 == 1) and not np.any(k == W.U64_MAX) and not np.any(v == W.U64_MAX)
    w3 = W.Workload(3, tree=1 << 14, batch=1 << 14)
    o, k, v = w3.batch_arrays(0)
    _, cnt = np.unique(k, return_counts=True)
    assert cnt.max() > 200          # zipf 0.99: the hottest key is hit ~5% of the time
    perm = W.scramble(np.arange(1000), 1000, 3)
    assert np.array_equal(np.sort(perm), np.arange(1000))
