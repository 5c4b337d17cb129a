"""Locality-aware warp reorganisation with a range field (RF): the paper's
iteration-warp traversal decisions, step by step (§5, P:1334-1512,
Fig.6) -- TEST INFRASTRUCTURE ONLY (same rules as the rest of oracle/: only
tests/, __graft_entry__.smoke() and bench.py's CPU legs may use it; it shares
nothing with the CUDA path).

Readings (SURVEY §8(c) reading 22):
  * RF(leaf) = the minimal key of the leaf `height` links to the right
    ("the minimal key of a node whose traversal steps from this
    node are tree height plus one"; the example -- height 5, RF(leaf 1) = min
    key of leaf 6 -- fixes the offset at `height` links); UINT64_MAX past the
    last leaf.
  * An iteration warp runs its request groups (RGs) in order with a buffer
    (leaf, RF).  The first RG, or an RG whose
    MAXIMAL key is larger than the buffered RF, traverses vertically
    (root to leaf: `height` nodes); otherwise horizontally along the leaf links
    from the buffered leaf.  After an RG the buffer holds the
    maximal leaf it accessed and that leaf's RF.
  * Traversal steps (Fig.10) of a request: `height` for a
    vertical traversal; 1 + the number of links followed for a horizontal one.
  * Lazy RF repair: a horizontal traversal that takes more than
    `height` steps sets RF(start leaf) to the min key of the leaf reached after
    `height` links.
"""
from __future__ import annotations

KEY_MAX = (1 << 64) - 1


def rf_table(leaf_min_keys: list[int], height: int) -> list[int]:
    """RF of every leaf of a leaf chain given in link order."""
    n = len(leaf_min_keys)
    return [leaf_min_keys[i + height] if i + height < n else KEY_MAX for i in range(n)]


def iteration_warp_plan(rg_keys: list[list[int]], leaf_of, rf: dict | list, height: int, leaf_min_keys=None):
    """Decisions of one iteration warp over its RGs (keys of each RG in SIMT
    order).  leaf_of(key) -> position of the key's leaf in the chain; rf maps
    a leaf position to its RF (mutated by the lazy repair when leaf_min_keys,
    the chain's min keys, is given).  Returns a list of dicts per RG:
    {"mode": "V"|"H", "buffer": leaf after the RG, "steps": [per request]}."""
    buf_leaf, buf_rf = None, None
    out = []
    for keys in rg_keys:
        kmax = max(keys)
        vertical = buf_leaf is None or kmax > buf_rf
        steps = []
        if vertical:
            steps = [height] * len(keys)
        else:
            start = buf_leaf
            for k in keys:
                target = leaf_of(k)
                s = 1 + max(0, target - start)
                steps.append(s)
                if s > height and leaf_min_keys is not None:
                    rf[start] = leaf_min_keys[start + height] if start + height < len(leaf_min_keys) else KEY_MAX
        top = leaf_of(kmax)
        buf_leaf, buf_rf = top, rf[top]
        out.append({"mode": "V" if vertical else "H", "buffer": top, "steps": steps})
    return out
