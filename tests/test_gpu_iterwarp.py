"""GPU: the paper's iteration warps + range field (EIRENE_F_ITERWARP, PAPER.md
§5) -- an ablation of the default query
traversal.  Two bars:

* results: bit-exact vs the oracle (the traversal mode never changes a
  result), over mixed batches that split leaves (stale, inherited RFs) and
  over the exhaustive tiny alphabet;
* decisions: on the pre-batch tree of a fresh bulk load, the kernel's count of
  vertical / horizontal request groups and its traversal steps equal the
  oracle's decision model (oracle/iterwarp.py) run over the same RGs --
  integers, exact.
"""
import numpy as np
import pytest
import torch

import oracle
from oracle.iterwarp import iteration_warp_plan, rf_table
from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W

pytestmark = pytest.mark.gpu


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


def _tree(dev, keys, vals, per=16, max_batch=1 << 16, **kw):
    from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree
    t = EireneTree(max_keys=max(1 << 12, 4 * len(keys)), max_batch=max_batch, iterwarp=True, **kw)
    if len(keys):
        t.bulk_load(T(keys, dev), T(vals, dev), leaf_fill=per / 16)
    return t


def _height(L):
    h, nc = 1, L
    while nc > 1:
        nc = (nc + 15) // 16
        h += 1
    return h


def _model(keys, per, q_list, w_list, iter_rgs):
    """Decision model over the bulk-loaded tree: RGs of 32 issued requests of the
    query list, then of the write list; iteration warp w runs RGs [w*I, (w+1)*I);
    the buffer empties where the write list starts."""
    L = (len(keys) + per - 1) // per
    height = _height(L)
    mins = [int(x) for x in keys[::per]]
    rf = rf_table(mins, height)

    def leaf_of(k):
        return max(0, int(np.searchsorted(keys, np.uint64(k), side="right")) - 1) // per

    rgs = [("q", q_list[i:i + 32]) for i in range(0, len(q_list), 32)] + \
          [("w", w_list[i:i + 32]) for i in range(0, len(w_list), 32)]
    vert = hor = steps = 0
    for w0 in range(0, len(rgs), iter_rgs):
        mine = rgs[w0:w0 + iter_rgs]
        for lst in ("q", "w"):
            part = [[int(x) for x in r] for tag, r in mine if tag == lst]
            if not part:
                continue
            for p in iteration_warp_plan(part, leaf_of, rf, height, mins):
                vert += p["mode"] == "V"
                hor += p["mode"] == "H"
                steps += sum(p["steps"])
    return vert, hor, steps


@pytest.mark.parametrize("per,iter_rgs,nkeys,n", [(16, 4, 1 << 14, 1 << 14), (11, 8, 1 << 13, 1 << 13),
                                                  (16, 1, 1 << 14, 1 << 12), (5, 3, 8000, 20000),
                                                  (16, 2, 1 << 16, 1 << 14)])
def test_decisions_match_the_oracle_model(dev, per, iter_rgs, nkeys, n):
    rng = np.random.default_rng(per * 1000 + iter_rgs)
    keys = np.unique(rng.integers(1, 1 << 40, size=2 * nkeys, dtype=np.uint64))[:nkeys] * np.uint64(2)
    vals = rng.integers(0, 1 << 62, size=keys.size, dtype=np.uint64)
    # queries of present and absent keys, updates, inserts: the query kernel sees the pre-batch tree
    ops = rng.choice(np.array([0, 1, 2, 3], np.uint8), size=n, p=[0.7, 0.1, 0.1, 0.1])
    k = np.where(rng.random(n) < 0.8, keys[rng.integers(0, keys.size, n)],
                 rng.integers(1, 1 << 41, n, dtype=np.uint64) | np.uint64(1))
    v = rng.integers(0, 1 << 62, size=n, dtype=np.uint64)
    t = _tree(dev, keys, vals, per=per, iter_rgs=iter_rgs)
    ref = oracle.MapOracle()
    ref.load(keys, vals)
    comb = oracle.combine_apply(ref, ops, k, v)
    isq = comb["issued_op"] == 0
    res, st = t.apply(T(ops, dev), T(k, dev), T(v, dev))
    assert np.array_equal(res.cpu().numpy(), comb["results"])
    vert, hor, steps = _model(keys, per, comb["issued_key"][isq], comb["issued_key"][~isq], iter_rgs)
    assert (st["rg_vertical"], st["rg_horizontal"], st["trav_steps"]) == (vert, hor, steps)
    if iter_rgs == 1:   # every RG is the first of its warp
        assert hor == 0 and steps == comb["n_issued"] * _height((len(keys) + per - 1) // per)
    elif nkeys <= n:   # >= 6 issued requests per leaf: an RG spans fewer leaves than the height
        assert hor > 0
    rk, rv = ref.scan()
    gk, gv = t.scan()
    assert np.array_equal(gk.cpu().numpy(), rk) and np.array_equal(gv.cpu().numpy(), rv)
    t.close()


@pytest.mark.parametrize("cfg_fracs,iter_rgs", [({W.QUERY: 0.5, W.INSERT: 0.5}, 0),
                                                ({W.QUERY: 0.3, W.INSERT: 0.6, W.DELETE: 0.1}, 4),
                                                ({W.QUERY: 0.95, W.UPDATE: 0.05}, 16)])
def test_results_over_split_batches(dev, cfg_fracs, iter_rgs):
    """Splits leave RFs stale (inherited by split-off leaves): results stay exact and
    later batches keep using horizontal traversals."""
    w = W.Workload(1, tree=1 << 14, batch=1 << 14, fracs=cfg_fracs)
    t = _tree(dev, w.keys, w.vals, iter_rgs=iter_rgs)
    ref = oracle.MapOracle()
    ref.load(w.keys, w.vals)
    for b in range(4):
        ops, keys, vals = w.batch_arrays(b)
        res, st = t.apply(T(ops, dev), T(keys, dev), T(vals, dev))
        want = ref.apply(ops, keys, vals)
        got = res.cpu().numpy()
        assert np.array_equal(got, want), f"batch {b}: {int(np.sum(got != want))} results differ"
        assert st["rg_vertical"] + st["rg_horizontal"] == \
            (st["issued_q"] + 31) // 32 + (st["issued_w"] + 31) // 32
        assert st["trav_steps"] >= st["issued_q"] + st["issued_w"]
    rk, rv = ref.scan()
    gk, gv = t.scan()
    assert np.array_equal(gk.cpu().numpy(), rk) and np.array_equal(gv.cpu().numpy(), rv)
    rc, nk = t.check_invariants()
    assert rc == 0 and nk == ref.size()
    t.close()


def test_growth_from_empty_tree(dev):
    """Root splits from a single empty leaf (RF = KEY_MAX inherited everywhere: every
    RG after the first is horizontal until a walk repairs its start)."""
    rng = np.random.default_rng(7)
    t = _tree(dev, np.empty(0, np.uint64), np.empty(0, np.uint64), iter_rgs=8)
    ref = oracle.MapOracle()
    for b in range(5):
        n = 1 << 13
        ops = rng.choice(np.array([0, 2, 3], np.uint8), size=n, p=[0.3, 0.6, 0.1])
        keys = rng.integers(1, 1 << 20, n, dtype=np.uint64)
        vals = rng.integers(0, 1 << 62, n, dtype=np.uint64)
        res, st = t.apply(T(ops, dev), T(keys, dev), T(vals, dev))
        want = ref.apply(ops, keys, vals)
        assert np.array_equal(res.cpu().numpy(), want), f"batch {b}"
    rk, rv = ref.scan()
    gk, gv = t.scan()
    assert np.array_equal(gk.cpu().numpy(), rk) and np.array_equal(gv.cpu().numpy(), rv)
    t.close()


def test_default_mode_reports_no_decisions(dev):
    rng = np.random.default_rng(3)
    keys = np.unique(rng.integers(1, 1 << 40, size=5000, dtype=np.uint64))
    t = _tree(dev, keys, keys)
    t.set_flags(iterwarp=False)
    ops = np.zeros(1000, np.uint8)
    k = keys[rng.integers(0, keys.size, 1000)]
    res, st = t.apply(T(ops, dev), T(k, dev), T(k, dev))
    assert np.array_equal(res.cpu().numpy(), k)
    assert st["trav_steps"] == 0 and st["rg_vertical"] == 0 and st["rg_horizontal"] == 0
    t.close()
