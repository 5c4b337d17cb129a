"""GPU parity of the 32-bit key / value build (libeirene32.so, -DEIRENE_KEY32;
SURVEY §8(f) NEXT(4): the paper's record width) against the CPU oracle,
bit-exact.  The oracle is width-agnostic (u64); a 32-bit NOT_FOUND (UINT32_MAX)
is compared as the oracle's NOT_FOUND."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W

pytestmark = pytest.mark.gpu
NF32 = np.uint32(0xFFFFFFFF)
NF64 = np.uint64(0xFFFFFFFFFFFFFFFF)


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ppopp_zhangz0lzl23_b200.build import build_all
    build_all()
    torch.cuda.set_device(0)
    return torch.device("cuda", 0)


def T32(a, dev):
    a = np.asarray(a)
    assert a.dtype == np.uint8 or int(a.max(initial=0)) <= 0xFFFFFFFF
    return torch.from_numpy(np.ascontiguousarray(a if a.dtype == np.uint8 else a.astype(np.uint32))).to(dev)


def widen(r):
    r = np.asarray(r).astype(np.uint64)
    r[r == np.uint64(0xFFFFFFFF)] = NF64
    return r


def tree32(dev, keys, vals, **kw):
    from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree
    t = EireneTree(key_bits=32, **kw)
    if len(keys):
        t.bulk_load(T32(keys, dev), T32(vals, dev))
    return t


def check(t, ref, ops, keys, vals, dev, scan=True):
    res, st = t.apply(T32(ops, dev), T32(keys, dev), T32(vals, dev))
    got = widen(res.cpu().numpy())
    want = ref.apply(ops, keys.astype(np.uint64), vals.astype(np.uint64))
    bad = np.nonzero(got != want)[0]
    assert bad.size == 0, f"{bad.size} differ, first {bad[:5]}: got {got[bad[:5]]} want {want[bad[:5]]}"
    if scan:
        k, v = t.scan()
        rk, rv = ref.scan()
        assert np.array_equal(k.cpu().numpy().astype(np.uint64), rk)
        assert np.array_equal(v.cpu().numpy().astype(np.uint64), rv)
    return st


def test_key32_bulk_load_scan(dev):
    w = W.Workload(7, tree=100000, batch=1024)
    assert int(w.keys.max()) < 0xFFFFFFFF and int(w.vals.max()) < 0xFFFFFFFF
    t = tree32(dev, w.keys, w.vals, max_keys=1 << 18, max_batch=1 << 12)
    k, v = t.scan()
    assert k.dtype == torch.uint32
    assert np.array_equal(k.cpu().numpy().astype(np.uint64), w.keys)
    assert np.array_equal(v.cpu().numpy().astype(np.uint64), w.vals)
    assert t.check_invariants() == (0, w.keys.size)
    t.close()


@pytest.mark.parametrize("dist", ["uniform", "zipf"])
def test_key32_mixed_batches(dev, dist):
    """Query / update / insert / delete batches with splits (and, Zipf, hot keys)."""
    w = W.Workload(7, tree=1 << 16, batch=1 << 15, dist=dist,
                   fracs={W.QUERY: 0.5, W.UPDATE: 0.2, W.INSERT: 0.25, W.DELETE: 0.05})
    t = tree32(dev, w.keys, w.vals, max_keys=1 << 19, max_batch=1 << 15)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    for b in range(4):
        ops, keys, vals = w.batch_arrays(b)
        st = check(t, ref, ops, keys, vals, dev, scan=(b == 3))
    assert st["leaf_splits"] > 0
    assert t.check_invariants() == (0, ref.size())
    t.close()


def test_key32_paper_default_shape(dev):
    """The u32 bench workload (cfg7: 2^23-key tree, 2^20 batches, 95/5 uniform) at full size."""
    w = W.Workload(7)
    t = tree32(dev, w.keys, w.vals, max_keys=1 << 24, max_batch=1 << 20)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    for b in range(2):
        ops, keys, vals = w.batch_arrays(b)
        check(t, ref, ops, keys, vals, dev, scan=(b == 1))
    t.close()


def test_key32_invalid_and_edges(dev):
    t = tree32(dev, np.array([5, 10], np.uint64), np.array([1, 2], np.uint64), max_keys=1 << 12, max_batch=64)
    ref = oracle.MapOracle(); ref.load(np.array([5, 10], np.uint64), np.array([1, 2], np.uint64))
    # extreme valid key / value: 2^32 - 2
    top = np.uint64(0xFFFFFFFE)
    check(t, ref, np.array([2, 0, 1, 0, 3, 0], np.uint8), np.array([top, top, 0, 0, top, top], np.uint64),
          np.array([top, 0, top, 0, 0, 0], np.uint64), dev)
    for ops, keys, vals in (([0], [0xFFFFFFFF], [0]), ([2], [7], [0xFFFFFFFF])):
        res = torch.empty(1, dtype=torch.uint32, device=dev)
        tk = t.submit(T32(np.array(ops, np.uint8), dev), T32(np.array(keys, np.uint64), dev),
                      T32(np.array(vals, np.uint64), dev), res)
        st = t.results(tk, raise_on_error=False)
        assert st["rc"] == -1
    k, v = t.scan()
    rk, rv = ref.scan()
    assert np.array_equal(k.cpu().numpy().astype(np.uint64), rk)
    t.close()


def test_key32_range_queries(dev):
    w = W.Workload(6, tree=1 << 14, batch=1 << 12, key_bits=32,
                   fracs={W.QUERY: 0.3, W.UPDATE: 0.2, W.INSERT: 0.1, W.DELETE: 0.1, W.RANGE: 0.3})
    t = tree32(dev, w.keys, w.vals, max_keys=1 << 16, max_batch=1 << 12)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    cap = 8
    for b in range(3):
        ops, keys, vals = w.batch_arrays(b)
        res, rk, rv, st = t.apply_range(T32(ops, dev), T32(keys, dev), T32(vals, dev), cap)
        want, wk, wv, _ = oracle.combine_apply_range(ref, ops, keys, vals, cap)
        got = widen(res.cpu().numpy())
        rng = ops == W.RANGE
        assert np.array_equal(got[rng], want[rng]) and np.array_equal(got[~rng], want[~rng])
        col = np.arange(cap)[None, :] < want.astype(np.int64)[:, None]
        col &= rng[:, None]
        assert np.array_equal(rk.cpu().numpy().astype(np.uint64)[col], wk[col])
        assert np.array_equal(rv.cpu().numpy().astype(np.uint64)[col], wv[col])
    t.close()


def test_key32_host_path(dev):
    w = W.Workload(7, tree=1 << 14, batch=1 << 12)
    t = tree32(dev, w.keys, w.vals, max_keys=1 << 16, max_batch=1 << 12)
    ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
    for b in range(3):
        ops, keys, vals = w.batch_arrays(b)
        pin = [torch.from_numpy(ops).pin_memory()] + [torch.from_numpy(a.astype(np.uint32)).pin_memory()
                                                        for a in (keys, vals)]
        hres = torch.empty(ops.size, dtype=torch.uint32).pin_memory()
        t.results(t.submit_host(*pin, hres))
        assert np.array_equal(widen(hres.numpy()), ref.apply(ops, keys, vals))
    t.close()
