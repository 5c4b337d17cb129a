"""Seeded synthetic workload generator.

This module is the ONLY code shared by the CUDA path's harness (tests, bench)
and the oracle side: it produces input arrays and holds none of the method's
arithmetic (no sorting of requests, no combining, no tree logic).

Workloads follow the paper's evaluation setup (§8.1):
YCSB-style request streams, uniform or Zipfian (theta = 0.99) keys, with the
paper's query/update mixes, but with u64 keys and values (BASELINE.json
configs[0]) instead of the paper's 32-bit records.

PRNG: counter-based splitmix64, x(seed, stream, i) = splitmix64(seed ^ (stream<<56) ^ i),
so any batch can be regenerated independently of the others.

Op codes (include/eirene.h): QUERY=0, UPDATE=1, INSERT=2, DELETE=3, RANGE=4.
A range request R(l, u) has key = l and val = u; the generator
picks l = loaded[j] and u = loaded[j + L - 1] so the range covers L loaded keys
("range query length" L of the paper's Fig.13).
Reserved sentinel: UINT64_MAX is never produced as a key or a write value.
"""
from __future__ import annotations

import numpy as np

QUERY, UPDATE, INSERT, DELETE, RANGE = 0, 1, 2, 3, 4
U64_MAX = np.uint64(0xFFFFFFFFFFFFFFFF)

# stream ids (top byte of the counter)
S_LOAD_KEY, S_LOAD_VAL, S_MIX, S_PICK, S_WVAL, S_FRESH, S_ZIPF, S_DEL, S_RANGE = 1, 2, 3, 4, 5, 6, 7, 8, 9

_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_G = np.uint64(0x9E3779B97F4A7C15)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser (Steele et al.); wraps mod 2^64."""
    with np.errstate(over="ignore"):
        z = x.astype(np.uint64) + _G
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def rand_u64(seed: int, stream: int, start: int, count: int) -> np.ndarray:
    base = np.uint64((seed ^ (stream << 56)) & 0xFFFFFFFFFFFFFFFF)
    idx = np.arange(start, start + count, dtype=np.uint64)
    return splitmix64(base ^ idx)


def uniform_index(x: np.ndarray, n: int) -> np.ndarray:
    """Lemire's multiply-shift: floor(x * n / 2^64), exact for n < 2^32."""
    assert 0 < n < (1 << 32)
    nn = np.uint64(n)
    with np.errstate(over="ignore"):
        xh = x >> np.uint64(32)
        xl = x & np.uint64(0xFFFFFFFF)
        return ((xh * nn + ((xl * nn) >> np.uint64(32))) >> np.uint64(32)).astype(np.int64)


def unit_double(x: np.ndarray) -> np.ndarray:
    return (x >> np.uint64(11)).astype(np.float64) * (1.0 / (1 << 53))


def sorted_unique(a: np.ndarray) -> np.ndarray:
    """== np.unique(a) for a 1-d integer array (sort + adjacent-difference mask;
    numpy 2.3's unique is ~15x slower on 2^24 u64)."""
    s = np.sort(a)
    if s.size < 2:
        return s
    keep = np.empty(s.size, dtype=bool)
    keep[0] = True
    np.not_equal(s[1:], s[:-1], out=keep[1:])
    return s[keep]


def loaded_keys(n: int, seed: int, key_bits: int = 64) -> tuple[np.ndarray, np.ndarray]:
    """n distinct EVEN keys (sorted) and their values (never the all-ones NOT_FOUND);
    key_bits 32: 32-bit keys and values (the u32 variant)."""
    keys = np.empty(0, dtype=np.uint64)
    start = 0
    while keys.size < n:
        need = n - keys.size
        draw = rand_u64(seed, S_LOAD_KEY, start, need + need // 64 + 16)
        if key_bits == 32:
            draw >>= np.uint64(32)
        draw &= ~np.uint64(1)
        start += draw.size
        keys = sorted_unique(np.concatenate([keys, draw]))
    if keys.size > n:
        # drop a seeded random subset so the kept keys stay uniform
        drop = np.argsort(rand_u64(seed, S_LOAD_KEY ^ 0x55, 0, keys.size))[: keys.size - n]
        keys = np.delete(keys, drop)
    vals = rand_u64(seed, S_LOAD_VAL, 0, n) >> np.uint64(1 if key_bits == 64 else 33)
    return keys, vals


def fresh_keys(seed: int, batch: int, count: int, key_bits: int = 64) -> np.ndarray:
    """Fresh insert keys: odd, so disjoint from the (even) loaded keys."""
    k = rand_u64(seed, S_FRESH, batch << 32, count)
    if key_bits == 32:
        k >>= np.uint64(32)
    k |= np.uint64(1)
    top = np.uint64(U64_MAX if key_bits == 64 else 0xFFFFFFFF)
    k[k == top] ^= np.uint64(2)
    return k


class Zipf:
    """YCSB / Gray et al. zipfian rank generator, theta in (0, 1), ranks in [0, n)."""

    def __init__(self, n: int, theta: float = 0.99):
        self.n, self.theta = n, theta
        zetan = 0.0
        chunk = 1 << 24
        for lo in range(1, n + 1, chunk):
            i = np.arange(lo, min(n + 1, lo + chunk), dtype=np.float64)
            zetan += float(np.sum(i ** -theta))
        self.zetan = zetan
        self.alpha = 1.0 / (1.0 - theta)
        zeta2 = 1.0 + 0.5 ** theta
        self.eta = (1.0 - (2.0 / n) ** (1.0 - theta)) / (1.0 - zeta2 / zetan)

    def ranks(self, u: np.ndarray) -> np.ndarray:
        uz = u * self.zetan
        r = (self.n * np.power(self.eta * u - self.eta + 1.0, self.alpha)).astype(np.int64)
        r = np.where(uz < 1.0 + 0.5 ** self.theta, 1, r)
        r = np.where(uz < 1.0, 0, r)
        return np.clip(r, 0, self.n - 1)


def scramble(rank: np.ndarray, n: int, seed: int) -> np.ndarray:
    """Seeded bijection on [0, n): odd-multiply + xorshift on the next power of two,
    cycle-walking back into [0, n)."""
    k = max(1, (n - 1).bit_length())
    mask = np.uint64((1 << k) - 1)
    a = np.uint64((0x9E3779B97F4A7C15 ^ (seed * 2)) | 1) & mask | np.uint64(1)
    b = np.uint64((0xD1B54A32D192ED03 ^ seed) | 1) & mask | np.uint64(1)
    s = np.uint64(max(1, k // 2))
    x = rank.astype(np.uint64)
    out = np.empty_like(x)
    todo = np.ones(x.shape, dtype=bool)
    cur = x.copy()
    with np.errstate(over="ignore"):
        while todo.any():
            y = (cur[todo] * a) & mask
            y = y ^ (y >> s)
            y = (y * b) & mask
            cur[todo] = y
            ok = todo.copy()
            ok[todo] = y < np.uint64(n)
            out[ok] = cur[ok]
            todo &= ~ok
    return out.astype(np.int64)


def shuffled_ops(n: int, fracs: dict[int, float], seed: int, batch: int) -> np.ndarray:
    """Exact counts round(p*n) per op type, then a seeded uniform shuffle
    (argsort of counter-based u64 draws)."""
    ops = np.empty(n, dtype=np.uint8)
    pos = 0
    items = sorted(fracs.items())
    for j, (op, p) in enumerate(items):
        cnt = n - pos if j == len(items) - 1 else int(round(p * n))
        ops[pos:pos + cnt] = op
        pos += cnt
    perm = np.argsort(rand_u64(seed, S_MIX, batch << 32, n), kind="stable")
    return ops[perm]


def make_batch(loaded: np.ndarray, n: int, fracs: dict[int, float], dist: str, seed: int,
               batch: int, zipf: Zipf | None = None, live: np.ndarray | None = None, range_len: int = 8,
               key_bits: int = 64):
    """One request batch: (ops u8[n], keys u64[n], vals u64[n]).

    QUERY/UPDATE keys are drawn from `loaded` (uniform or scrambled Zipf);
    INSERT keys are fresh odd keys; DELETE keys are uniform over `live`
    (the live-key snapshot at batch start, with replacement)."""
    ops = shuffled_ops(n, fracs, seed, batch)
    keys = np.empty(n, dtype=np.uint64)
    x = rand_u64(seed, S_PICK, batch << 32, n)
    m = len(loaded)
    sel = (ops == QUERY) | (ops == UPDATE)
    if dist == "uniform":
        idx = uniform_index(x[sel], m)
    elif dist == "zipf":
        assert zipf is not None and zipf.n == m
        idx = scramble(zipf.ranks(unit_double(x[sel])), m, seed)
    else:
        raise ValueError(dist)
    keys[sel] = loaded[idx]
    ins = ops == INSERT
    keys[ins] = fresh_keys(seed, batch, int(ins.sum()), key_bits)
    dele = ops == DELETE
    if dele.any():
        pool = live if live is not None else loaded
        keys[dele] = pool[uniform_index(rand_u64(seed, S_DEL, batch << 32, int(dele.sum())), len(pool))]
    vals = rand_u64(seed, S_WVAL, batch << 32, n) >> np.uint64(1 if key_bits == 64 else 33)
    vals[ops == QUERY] = 0
    rng_ = ops == RANGE
    if rng_.any():
        L = max(1, min(range_len, m))
        j = uniform_index(rand_u64(seed, S_RANGE, batch << 32, int(rng_.sum())), m - L + 1)
        keys[rng_] = loaded[j]
        vals[rng_] = loaded[j + L - 1]
    return ops, keys, vals


# ---------------------------------------------------------------- configs
# BASELINE.json configs[0..4] == cfg1..cfg5; seed = 0xE1E2E3E4 + cfg.
CONFIGS = {
    # per_tree: steps per freshly bulk-loaded tree in the bench (cfg1 one batch
    # per fresh tree, cfg4 ~4 insert-heavy batches per seed until >= 2^22 live keys)
    1: dict(tree=1 << 16, batch=1 << 16, fracs={QUERY: 0.5, INSERT: 0.5}, dist="uniform", per_tree=1),
    2: dict(tree=1 << 24, batch=1 << 20, fracs={QUERY: 0.95, UPDATE: 0.05}, dist="uniform"),
    3: dict(tree=1 << 24, batch=1 << 20, fracs={QUERY: 0.5, UPDATE: 0.5}, dist="zipf"),
    4: dict(tree=1 << 20, batch=1 << 20, fracs={INSERT: 0.9, DELETE: 0.1}, dist="uniform", per_tree=4),
    5: dict(tree=1 << 28, batch=1 << 24, fracs={QUERY: 0.95, UPDATE: 0.05}, dist="zipf", strong=True),
    # the paper's pure range-query workload (Fig.13), length 8
    6: dict(tree=1 << 24, batch=1 << 20, fracs={RANGE: 1.0}, dist="uniform", range_len=8),
    # the paper's default workload with its record width -- 32-bit keys and
    # values, 2^23-key tree, 1M-request batches, 95% query / 5% update, uniform
    7: dict(tree=1 << 23, batch=1 << 20, fracs={QUERY: 0.95, UPDATE: 0.05}, dist="uniform", key_bits=32),
}


# YCSB-like mixes of cfg5 (BASELINE configs[4]): workload A
# (50% read / 50% update, Zipf), B (95 / 5, Zipf), C (100% read, Zipf) and the
# paper's default 95 / 5 uniform
MIXES = {
    "A": (dict({0: 0.5, 1: 0.5}), "zipf"),
    "B": (dict({0: 0.95, 1: 0.05}), "zipf"),
    "C": (dict({0: 1.0}), "zipf"),
    "U": (dict({0: 0.95, 1: 0.05}), "uniform"),
}


def seed_for(cfg: int) -> int:
    return 0xE1E2E3E4 + cfg


class Workload:
    """Generates the bulk-load arrays and a stream of batches for one config,
    optionally scaled down (tree/batch sizes overridden) for parity tests."""

    def __init__(self, cfg: int, tree: int | None = None, batch: int | None = None,
                 fracs: dict | None = None, dist: str | None = None, seed: int | None = None,
                 range_len: int | None = None, key_bits: int | None = None):
        c = dict(CONFIGS[cfg])
        self.key_bits = key_bits or c.get("key_bits", 64)
        self.range_len = range_len or c.get("range_len", 8)
        self.cfg = cfg
        self.tree = tree or c["tree"]
        self.batch = batch or c["batch"]
        self.fracs = fracs or c["fracs"]
        self.dist = dist or c["dist"]
        self.seed = seed_for(cfg) if seed is None else seed
        self.keys, self.vals = loaded_keys(self.tree, self.seed, self.key_bits)
        self.zipf = Zipf(self.tree) if self.dist == "zipf" else None
        self.live = self.keys if DELETE in self.fracs else None

    def batch_arrays(self, b: int):
        ops, keys, vals = make_batch(self.keys, self.batch, self.fracs, self.dist, self.seed, b,
                                     zipf=self.zipf, live=self.live, range_len=self.range_len, key_bits=self.key_bits)
        if self.live is not None:
            # live-key snapshot for the next batch (generator bookkeeping only)
            ins = keys[ops == INSERT]
            dele = keys[ops == DELETE]
            self.live = np.setdiff1d(np.union1d(self.live, ins), dele)
        return ops, keys, vals
