"""CPU checks of bench.py's measurement arithmetic: the counts
behind the random-access roofline and the query kernel's algorithmic bytes,
against brute force over a tiny bulk-loaded shape."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W  # noqa: E402


def _brute(loaded, ops, keys, per):
    """Leaf / sector touches by walking the issued requests one by one."""
    issued = {}
    for o, k in zip(ops.tolist(), keys.tolist()):
        issued[k] = issued.get(k, False) or o != W.QUERY   # issued write iff any write
    lines, sectors, qlines, qsectors = set(), set(), set(), set()
    pos_of = {int(k): i for i, k in enumerate(loaded.tolist())}
    for k, w in issued.items():
        p = int(np.searchsorted(loaded, np.uint64(k)))
        leaf = p // per
        lines.add(leaf)
        if not w:
            qlines.add(leaf)
        if k in pos_of:
            sectors.add((leaf, (pos_of[k] % per) // 4))
            if not w:
                qsectors.add((leaf, (pos_of[k] % per) // 4))
    nw = sum(1 for w in issued.values() if w)
    return lines, sectors, nw, qlines, qsectors, len(issued) - nw


def test_random_access_counts_brute_force():
    rng = np.random.default_rng(3)
    loaded = np.unique(rng.integers(1, 1 << 30, 3000, dtype=np.uint64)) * np.uint64(2)
    n = 2000
    ops = rng.choice(np.array([0, 1, 2, 3], np.uint8), n, p=[0.6, 0.2, 0.1, 0.1])
    keys = np.where(rng.random(n) < 0.8, loaded[rng.integers(0, loaded.size, n)],
                    rng.integers(1, 1 << 31, n, dtype=np.uint64) | np.uint64(1)).astype(np.uint64)
    c = bench.random_access_counts(loaded, ops, keys, 16)
    lines, sectors, nw, *_ = _brute(loaded, ops, keys, 16)
    assert c["lines"] * n == len(lines)
    assert c["sectors"] * n == len(sectors)
    assert c["writes"] * n == nw
    ups = int(np.sum((ops == W.UPDATE) | (ops == W.INSERT)))
    assert c["bio"] * n == n * 17 + 8 * ups


def test_query_algorithmic_bytes_brute_force():
    rng = np.random.default_rng(4)
    loaded = np.unique(rng.integers(1, 1 << 30, 5000, dtype=np.uint64))
    n = 3000
    ops = rng.choice(np.array([0, 1], np.uint8), n, p=[0.9, 0.1])
    keys = loaded[rng.integers(0, loaded.size, n)]
    ab = bench.algorithmic_bytes_query(loaded, ops, keys, 16)
    _, _, _, qlines, qsectors, nq = _brute(loaded, ops, keys, 16)
    assert ab["issued_q"] == nq and ab["leaf_lines"] == len(qlines) and ab["value_sectors"] == len(qsectors)
    assert ab["bytes"] == nq * 20 + len(qlines) * 128 + len(qsectors) * 32
