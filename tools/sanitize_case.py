"""Small batches for compute-sanitizer runs (tools/sanitize.sh): the STM path
(FORCE_STM, THRESHOLD 0) on a split-heavy insert/delete mix, and a 2^12-key
cfg1-shaped batch (every leaf splits), both checked against the oracle."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import oracle  # noqa: E402
from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W  # noqa: E402
from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree  # noqa: E402


def T(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def check(t, ref, ops, ks, vs):
    res, st = t.apply(T(ops), T(ks), T(vs))
    assert np.array_equal(res.cpu().numpy(), ref.apply(ops, ks, vs)), "results differ"
    return st


def main(which):
    rng = np.random.default_rng(17)
    if which in ("stm", "all"):
        keys = np.unique(rng.integers(1, 1 << 20, 6000, dtype=np.uint64))[:3000]
        vals = rng.integers(0, 1 << 62, keys.size, dtype=np.uint64)
        t = EireneTree(max_keys=1 << 14, max_batch=1 << 12, retry_threshold=0, force_stm=True)
        t.bulk_load(T(keys), T(vals))
        ref = oracle.MapOracle(); ref.load(keys, vals)
        for b in range(2):
            n = 1 << 12
            ops = rng.choice(np.array([0, 1, 2, 3], np.uint8), n, p=[0.3, 0.2, 0.4, 0.1])
            ks = np.where(rng.random(n) < 0.5, keys[rng.integers(0, keys.size, n)],
                          rng.integers(1, 1 << 20, n, dtype=np.uint64)).astype(np.uint64)
            vs = rng.integers(0, 1 << 62, n, dtype=np.uint64)
            st = check(t, ref, ops, ks, vs)
            assert st["stm_fallbacks"] > 0
        assert t.check_invariants()[0] == 0
        t.close()
        print("stm case ok")
    if which in ("cfg1", "all"):
        w = W.Workload(1, tree=1 << 12, batch=1 << 12)
        t = EireneTree(max_keys=1 << 14, max_batch=1 << 12)
        t.bulk_load(T(w.keys), T(w.vals))
        ref = oracle.MapOracle(); ref.load(w.keys, w.vals)
        st = check(t, ref, *w.batch_arrays(0))
        assert st["leaf_splits"] > 0
        assert t.check_invariants()[0] == 0
        t.close()
        print("cfg1 case ok")


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "all")
