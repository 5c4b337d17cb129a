"""Pins for the range-query part of the CPU oracle (
PAPER.md §4.1.2).  Runs without a GPU.

A range request R(l, u) (op RANGE = 4, key = l, val = u, inclusive) returns
the pairs of the state visible just before it with l <= k <= u, ascending,
limited to the first `cap` (readings R1-R3).  The pins:
  * the paper's Fig.4 and Fig.5 worked examples (tests/golden/fig4.json,
    fig5.json), including the number of artificial queries of Fig.5;
  * a range-only batch == slices of the loaded sorted arrays (numpy
    searchsorted), any cap;
  * engine (iii) -- the paper's artificial-query mechanism, a different
    algorithm -- agrees with engine (i), the definition, by exhaustive
    enumeration of tiny sequences and on random conflict-heavy batches;
  * the artificial-query count equals its closed form (pairs (R, k) with k in
    [l, u] and k written in the batch);
  * engine (ii) (B+tree leaf-chain walk, small fanouts) agrees with (i).
"""
import itertools
import json
import os

import numpy as np
import pytest

from oracle import NOT_FOUND, RANGE, BTreeOracle, MapOracle, combine_apply_range

OPC = {"Q": 0, "U": 1, "I": 2, "D": 3, "R": RANGE}
NF = int(NOT_FOUND)


def _load_fig(golden_dir, name):
    with open(os.path.join(golden_dir, name)) as f:
        g = json.load(f)
    val = g["values"]
    pk = np.array([k for k, _ in g["pre_batch"]], dtype=np.uint64)
    pv = np.array([val[v] for _, v in g["pre_batch"]], dtype=np.uint64)
    reqs = sorted(g["requests"], key=lambda r: r["ts"])
    ts_index = {r["ts"]: i for i, r in enumerate(reqs)}   # relabel timestamps to batch indices
    ops = np.array([OPC[r["op"]] for r in reqs], np.uint8)
    keys = np.array([r["lo"] if r["op"] == "R" else r["key"] for r in reqs], np.uint64)
    vals = np.array([r["hi"] if r["op"] == "R" else val.get(r.get("val"), 0) for r in reqs], np.uint64)
    return g, val, pk, pv, ops, keys, vals, ts_index


def _engines():
    return {
        "map": lambda: MapOracle(),
        "bt3": lambda: BTreeOracle(3),
        "bt16": lambda: BTreeOracle(16),
    }


def _run(engine, pk, pv, ops, keys, vals, cap):
    if engine == "comb":
        m = MapOracle()
        m.load(pk, pv)
        res, rk, rv, nart = combine_apply_range(m, ops, keys, vals, cap)
        return res, rk, rv, m, nart
    e = _engines()[engine]()
    e.load(pk, pv)
    res, rk, rv = e.apply_range(ops, keys, vals, cap)
    return res, rk, rv, e, None


@pytest.mark.parametrize("engine", ["map", "bt3", "bt16", "comb"])
@pytest.mark.parametrize("fig", ["fig4.json", "fig5.json"])
def test_paper_range_examples(golden_dir, fig, engine):
    g, val, pk, pv, ops, keys, vals, tsi = _load_fig(golden_dir, fig)
    cap = 8
    res, rk, rv, e, nart = _run(engine, pk, pv, ops, keys, vals, cap)
    for part in ("expected_range_paper", "expected_range_reading"):
        for ts, kv in g.get(part, {}).items():
            if ts.startswith("_"):
                continue
            i = tsi[int(ts)]
            got = {int(rk[i, j]): int(rv[i, j]) for j in range(int(res[i]))}
            for k, v in kv.items():
                assert got.get(int(k)) == val[v], f"{fig} R@T{ts} key {k}: got {got.get(int(k))}, want {val[v]}"
            if part == "expected_range_reading" or fig == "fig5.json":
                assert len(got) == len(kv)
    for ts, v in g.get("expected_results_paper", {}).items():
        if not ts.startswith("_"):
            assert int(res[tsi[int(ts)]]) == val[v]
    k, v = e.scan()
    assert [(int(a), int(b)) for a, b in zip(k, v)] == [(kk, val[vv]) for kk, vv in g["final_state"]]
    if engine == "comb" and "artificial_queries" in g:
        assert nart == g["artificial_queries"]["count"]


@pytest.mark.parametrize("engine", ["map", "bt3", "bt16", "comb"])
@pytest.mark.parametrize("cap", [1, 4, 16, 64])
def test_range_only_batch_is_sorted_slice(engine, cap):
    """Special case: with no writes, R(l, u) == the slice [searchsorted(l, left),
    searchsorted(u, right)) of the loaded sorted arrays, first cap of it."""
    rng = np.random.default_rng(21)
    keys = np.unique(rng.integers(0, 1 << 30, 3000, dtype=np.uint64))
    vals = rng.integers(0, 1 << 62, keys.size, dtype=np.uint64)
    n = 500
    lo = rng.integers(0, 1 << 30, n, dtype=np.uint64)
    span = rng.integers(0, 1 << 22, n, dtype=np.uint64)
    hi = lo + span
    hi[:20] = lo[:20] - 1                    # empty (l > u)
    hi[20:40] = np.uint64(NF)                # unbounded above
    lo[40:60] = keys[rng.integers(0, keys.size, 20)]   # bounds on existing keys (inclusive)
    hi[40:60] = lo[40:60]
    res, rk, rv, _, _ = _run(engine, keys, vals, np.full(n, RANGE, np.uint8), lo, hi, cap)
    for i in range(n):
        a = np.searchsorted(keys, lo[i], "left")
        b = np.searchsorted(keys, hi[i], "right") if hi[i] >= lo[i] else a
        c = min(cap, max(0, b - a))
        assert int(res[i]) == c
        assert np.array_equal(rk[i, :c], keys[a:a + c]) and np.array_equal(rv[i, :c], vals[a:a + c])


def _art_count(ops, keys, vals):
    wk = set(int(k) for o, k in zip(ops, keys) if o in (1, 2, 3))
    return sum(sum(1 for k in wk if int(l) <= k <= int(u)) for o, l, u in zip(ops, keys, vals) if o == RANGE)


def test_exhaustive_tiny_with_ranges():
    """Brute force: every sequence of length <= 3 over 3 keys with
    {Q, U, D} per key plus the ranges [10,20], [20,30], [10,30], [15,15]
    (13 choices per position), from 4 initial states: engine (iii) (the
    paper's mechanism) == engine (i) (the definition), cap 1 and 3."""
    alphabet = [(op, k, v) for k in (10, 20, 30) for (op, v) in ((0, 0), (1, 7), (3, 0))]
    alphabet += [(RANGE, 10, 20), (RANGE, 20, 30), (RANGE, 10, 30), (RANGE, 15, 15)]
    inits = [{}, {10: 1}, {20: 2, 30: 3}, {10: 1, 20: 2, 30: 3}]
    count = 0
    for init in inits:
        ik = np.array(sorted(init), dtype=np.uint64)
        iv = np.array([init[k] for k in sorted(init)], dtype=np.uint64)
        for L in range(1, 4):
            for seq in itertools.product(alphabet, repeat=L):
                ops = np.array([s[0] for s in seq], np.uint8)
                keys = np.array([s[1] for s in seq], np.uint64)
                vals = np.array([s[2] for s in seq], np.uint64)
                for cap in (1, 3):
                    a = _run("map", ik, iv, ops, keys, vals, cap)
                    c = _run("comb", ik, iv, ops, keys, vals, cap)
                    for x, y in zip(a[:3], c[:3]):
                        assert np.array_equal(x, y), (init, seq, cap)
                    assert np.array_equal(a[3].scan()[0], c[3].scan()[0])
                    assert c[4] == _art_count(ops, keys, vals)
                count += 1
    assert count == 4 * sum(13 ** L for L in range(1, 4))


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_comb_range_vs_definition_random(seed):
    """Random conflict-heavy batches mixing every op with ranges of random
    width; several batches in sequence (state carried)."""
    rng = np.random.default_rng(300 + seed)
    keys = np.unique(rng.integers(0, 600, 300, dtype=np.uint64))
    vals = rng.integers(0, 1 << 62, keys.size, dtype=np.uint64)
    engines = [_engines()["map"](), _engines()["bt3"](), MapOracle()]
    for e in engines:
        e.load(keys, vals)
    for b in range(20):
        n = int(rng.integers(1, 800))
        ops = rng.integers(0, 5, n).astype(np.uint8)
        ks = rng.integers(0, 600, n, dtype=np.uint64)
        vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
        r = ops == RANGE
        vs[r] = ks[r] + rng.integers(0, 80, int(r.sum()), dtype=np.uint64)
        cap = int(rng.integers(1, 40))
        a = engines[0].apply_range(ops, ks, vs, cap)
        t = engines[1].apply_range(ops, ks, vs, cap)
        c = combine_apply_range(engines[2], ops, ks, vs, cap)
        for x, y, z in zip(a, t, c[:3]):
            assert np.array_equal(x, y) and np.array_equal(x, z)
        assert engines[1].check() == 0
        assert c[3] == _art_count(ops, ks, vs)
    for x, y in zip(engines[0].scan(), engines[2].scan()):
        assert np.array_equal(x, y)


def test_range_results_are_snapshots():
    """Invariant: a range's pairs equal a point query of each key at the same
    timestamp (the range is a consistent snapshot), and every key of the
    snapshot inside [l, u] is reported up to cap."""
    rng = np.random.default_rng(5)
    keys = np.unique(rng.integers(0, 200, 100, dtype=np.uint64))
    vals = rng.integers(0, 1000, keys.size, dtype=np.uint64)
    n = 300
    ops = rng.integers(0, 5, n).astype(np.uint8)
    ks = rng.integers(0, 200, n, dtype=np.uint64)
    vs = rng.integers(0, 1000, n, dtype=np.uint64)
    r = ops == RANGE
    vs[r] = ks[r] + 30
    cap = 64
    m = MapOracle(); m.load(keys, vals)
    res, rk, rv = m.apply_range(ops, ks, vs, cap)
    for i in np.nonzero(r)[0]:
        q = MapOracle(); q.load(keys, vals)
        q.apply(ops[:i][ops[:i] != RANGE], ks[:i][ops[:i] != RANGE], vs[:i][ops[:i] != RANGE])
        sk, sv = q.scan(int(ks[i]), int(vs[i]))
        c = int(res[i])
        assert c == min(cap, sk.size)
        assert np.array_equal(rk[i, :c], sk[:c]) and np.array_equal(rv[i, :c], sv[:c])


def test_invalid_point_request_in_range_batch():
    m = MapOracle()
    with pytest.raises(ValueError):
        m.apply_range(np.array([5], np.uint8), np.array([1], np.uint64), np.array([2], np.uint64), 4)
    with pytest.raises(ValueError):
        m.apply_range(np.array([1], np.uint8), np.array([NF], np.uint64), np.array([2], np.uint64), 4)
    # a range may use UINT64_MAX as its bounds
    res, _, _ = m.apply_range(np.array([RANGE], np.uint8), np.array([NF], np.uint64), np.array([NF], np.uint64), 4)
    assert int(res[0]) == 0
