#!/usr/bin/env python
"""Benchmark of the Eirene batched B+tree hot path on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 2] [--impl ours|reference]

One step = one batch through the whole hot path (sort -> combine -> partition ->
query -> update -> RESULT_CAL) on synthetic YCSB-style input
(workload.py, BASELINE.json configs).  N=1 workload = configs[1] (cfg2): 2^24
u64 keys, 2^20-request batches, 95% query / 5% update, uniform keys.  With
N > 1 (torchrun, one rank per GPU, NCCL) the tree is range-partitioned and
every rank routes its timestamp slice of each global batch with all-to-all
(weak scaling: 2^24 keys and 2^20 requests per GPU).

Prints ONE JSON line on rank 0 (see DESIGN.md §6 for every field).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W  # noqa: E402

PEAKS_FALLBACK = {"hbm_gbs": 6650.0, "source": "fallback (B200_PROFILING.md)"}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return {"hbm_gbs": float(d["hbm_gbs"]), "source": "measured (MEASURED_PEAKS.json)"}
    except Exception:
        return dict(PEAKS_FALLBACK)


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        sm = [float(r[1]) for r in self.rows if len(r) > 2 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) > 2 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for i, nm in enumerate(names):
                if len(r) > 5 + i and r[5 + i].lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


# --------------------------------------------------------------------------- stats
def spread(ms: np.ndarray, source: str) -> dict:
    """Per-batch response time summary: the paper's "variance" (max - min) / mean
    (reading 24) and the coefficient of variation beside it."""
    ms = np.asarray(ms, dtype=np.float64)
    return {"mean": float(ms.mean()), "min": float(ms.min()), "max": float(ms.max()),
            "variance_maxmin_over_mean": float((ms.max() - ms.min()) / ms.mean()),
            "cv": float(ms.std() / ms.mean()), "n": int(ms.size), "source": source}



def algorithmic_bytes_query(loaded: np.ndarray, ops: np.ndarray, keys: np.ndarray, per_leaf: int,
                            kb: int = 8) -> dict:
    """Algorithmic HBM bytes of the QUERY kernel for one cfg2 batch:
    per issued query 8 B key + 4 B seg read + 8 B result write, one 128 B leaf key
    line per distinct leaf touched, one 32 B value sector per distinct (leaf, sector)
    hit.  Valid for batches on the bulk-loaded shape (cfg2 never splits).  kb = bytes per key
    and value (8; 4 for the 32-bit build: a 64 B key line, 8 values per sector)."""
    uk = W.sorted_unique(keys)
    issued_w = np.zeros(uk.size, bool)
    w = ops != W.QUERY
    # a key issues a write iff any write on it
    wk = W.sorted_unique(keys[w])
    issued_w[np.searchsorted(uk, wk)] = True
    qk = uk[~issued_w]
    pos = np.searchsorted(loaded, qk)
    hit = (pos < loaded.size) & (loaded[np.minimum(pos, loaded.size - 1)] == qk)
    leaf = pos // per_leaf
    slot = pos % per_leaf
    lines = W.sorted_unique(leaf).size
    vps = 32 // kb
    sectors = W.sorted_unique(leaf[hit] * 4 + slot[hit] // vps).size
    nq = qk.size
    return {"issued_q": int(nq), "leaf_lines": int(lines), "value_sectors": int(sectors),
            "bytes": int(nq * (kb + 4 + kb) + lines * 16 * kb + sectors * 32)}


def algorithmic_bytes_range(loaded: np.ndarray, ops: np.ndarray, keys: np.ndarray, vals: np.ndarray,
                            per_leaf: int, cap: int) -> dict:
    """Algorithmic HBM bytes of the RANGE kernel for one range-only batch on the
    bulk-loaded shape (no writes): per range 1 B op + 8 B l + 8 B u read, 8 B
    count + 16 B per returned pair written; one 128 B leaf key line per distinct
    leaf the walks touch and one 32 B value sector per distinct (leaf, sector)
    returned.  Inner levels are L2-resident (not counted)."""
    r = ops == W.RANGE
    lo = np.searchsorted(loaded, keys[r], "left")
    hi = np.searchsorted(loaded, vals[r], "right")
    cnt = np.minimum(np.maximum(hi - lo, 0), cap)
    idx = np.concatenate([np.arange(a, a + c) for a, c in zip(lo, cnt)]) if cnt.size else np.empty(0, np.int64)
    leaf = idx // per_leaf
    # the walk reads the leaf of l even when it holds no key of the range
    lines = W.sorted_unique(np.concatenate([leaf, np.minimum(lo, loaded.size - 1) // per_leaf])).size
    sectors = W.sorted_unique(leaf * 4 + (idx % per_leaf) // 4).size
    nr = int(r.sum())
    return {"ranges": nr, "pairs": int(cnt.sum()), "leaf_lines": int(lines), "value_sectors": int(sectors),
            "bytes": int(nr * (1 + 8 + 8 + 8) + int(cnt.sum()) * 16 + lines * 128 + sectors * 32)}


def random_access_counts(loaded: np.ndarray, ops: np.ndarray, keys: np.ndarray, per_leaf: int,
                         kb: int = 8) -> dict:
    """Random HBM touches of one batch on the bulk-loaded shape:
    every issued request (one per distinct key, query or write) reads its leaf's
    128 B key line (distinct leaves counted once) and, if its key is present,
    one 32 B value sector (distinct sectors once); every issued write writes
    one 32 B value sector.  Streamed bytes per request: op 1 + key 8 +
    result 8, + 8 per upsert value."""
    uk = W.sorted_unique(keys)
    wk = W.sorted_unique(keys[ops != W.QUERY])
    pos = np.searchsorted(loaded, uk)
    hit = (pos < loaded.size) & (loaded[np.minimum(pos, loaded.size - 1)] == uk)
    leaf = pos // per_leaf
    n = keys.size
    ups = int(np.sum((ops == W.UPDATE) | (ops == W.INSERT)))
    vps = 32 // kb
    return {"lines": W.sorted_unique(leaf).size / n,
            "sectors": W.sorted_unique(leaf[hit] * 4 + (pos[hit] % per_leaf) // vps).size / n,
            "writes": wk.size / n, "bio": (n * (1 + 2 * kb) + ups * kb) / n, "line_bytes": 16 * kb}


def probe_random_access(dev, stream, pool_bytes: int, n: int = 1 << 24, n_leaf: int = 1 << 20,
                        reps: int = 3) -> dict:
    """Random accesses per second of this GPU's HBM (eirene_probe_gather) over a
    pool the size of the leaf pool (power of two >= the tree's leaf blocks, so the
    TLB reach matches): R128 = 128 B line reads, R32 = 32 B sector reads, R32w =
    32 B sector writes (uniformly random), R_leaf = the query kernel's leaf access
    (key line + dependent value sector of a 256 B block) at a key-sorted batch's
    order and density (n_leaf blocks visited ascending).  Best of `reps`, CUDA
    events on the launching stream."""
    import ctypes

    import torch

    from paper_conf_ppopp_zhangz0lzl23_b200 import _ffi
    L = _ffi.lib()
    pool = torch.empty(pool_bytes, dtype=torch.uint8, device=dev)
    out = {"pool_bytes": pool_bytes}
    for kind, name, cnt in ((0, "R128", n), (1, "R32", n), (2, "R32w", n), (3, "R_leaf", n_leaf)):
        best = 0.0
        for r in range(reps + 1):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            rc = L.eirene_probe_gather(ctypes.c_void_p(pool.data_ptr()), pool.numel(), cnt, kind, 77 + r,
                                       ctypes.c_void_p(stream.cuda_stream))
            e1.record(stream)
            stream.synchronize()
            if rc != 0:
                raise RuntimeError(f"eirene_probe_gather rc={rc}")
            if r:   # first launch is a warm-up
                best = max(best, cnt / (e0.elapsed_time(e1) * 1e-3))
        out[name] = best
    del pool
    return out


def run_reference(args):
    """--impl reference: the CPU oracle (sequential B+tree, 1 thread) as it stands,
    each step a bounded sample of the same workload."""
    import oracle
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    cfg = args.config
    wl = W.Workload(cfg)
    t = oracle.BTreeOracle(16)
    t0 = time.time()
    t.load(wl.keys, wl.vals)
    load_s = time.time() - t0
    sample = args.ref_sample
    times = []
    total = 0
    cap = W.CONFIGS[cfg].get("range_len", 0)
    for s in range(args.warmup + args.steps):
        ops, keys, vals = wl.batch_arrays(s)
        ops, keys, vals = ops[:sample], keys[:sample], vals[:sample]
        with pinned_core():
            a = time.perf_counter()
            if cap:
                t.apply_range(ops, keys, vals, cap)
            else:
                t.apply(ops, keys, vals)
            dt = time.perf_counter() - a
        if s >= args.warmup:
            times.append(dt)
            total += sample
    tt = sum(times)
    v = total / tt / 1e9
    line = {
        "impl": "reference", "metric": "requests/sec per batch", "value": v, "unit": "Greq/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tt / len(times),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": {"workload": f"cfg{cfg}: {W.CONFIGS[cfg]['tree']} keys, batch sample {sample} of "
                               f"{W.CONFIGS[cfg]['batch']} requests", "cfg": cfg},
        "cpu_baseline": {"value": v, "unit": "Greq/s", "cores": 1, "host_cores": os.cpu_count(), "kind": "oracle",
                         "sample": f"{args.steps} batches x first {sample} requests; oracle B+tree bulk load "
                                   f"{load_s:.1f}s untimed"},
        "e2e": {"value": v, "unit": "Greq/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def slice_parity(wl, got_batches, splitters, slice_keys: int) -> dict:
    """Bit-exact check of the first global batches on key slices (see the caller)."""
    import oracle
    K, V = wl.keys, wl.vals
    starts = [0, max(0, K.size - slice_keys)]
    for s in splitters:
        starts.append(int(np.clip(np.searchsorted(K, s) - slice_keys // 2, 0, max(0, K.size - slice_keys))))
    starts = sorted(set(starts))
    bad = checked = 0
    for a in starts:
        b = min(K.size, a + slice_keys)
        lo = int(K[a]) if a > 0 else 0
        hi = int(K[b]) if b < K.size else None
        ref = oracle.MapOracle()
        ref.load(K[a:b], V[a:b])
        for bi, got in enumerate(got_batches):
            o, k, v = wl.batch_arrays(bi)
            m = (k >= np.uint64(lo)) & ((k < np.uint64(hi)) if hi is not None else True)
            want = ref.apply(o[m], k[m], v[m])
            bad += int(np.sum(got[m] != want))
            checked += int(m.sum())
    return {"batches_checked": len(got_batches), "requests_checked": checked, "mismatches": bad,
            "vs": f"oracle (std::map) on {len(starts)} key slices of {slice_keys} loaded keys (one across every "
                  f"shard boundary, both ends), every request of the slice, bit-exact"}


def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.gpus != world and world > 1:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE {world}")
    # --backend gloo / EIRENE_BENCH_ONE_GPU=1: functional check of the N>1 code
    # path with every rank on cuda:0 (NCCL needs one GPU per rank); never a
    # number to report
    if os.environ.get("EIRENE_BENCH_ONE_GPU"):
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(args.backend)
        from paper_conf_ppopp_zhangz0lzl23_b200.parallel import ShardedEirene
    cfg = args.config
    C = dict(W.CONFIGS[cfg])
    if args.mix:   # YCSB-like mix override (cfg5: A, B, C, U)
        C["fracs"], C["dist"] = W.MIXES[args.mix]
    wkw = {"fracs": C["fracs"], "dist": C["dist"]}
    # cfg7: the 32-bit key / value build, libeirene32.so
    kbits = C.get("key_bits", 64)
    kb = kbits // 8
    kdt = torch.uint32 if kbits == 32 else torch.uint64
    if kbits == 32 and world > 1:
        raise SystemExit("the 32-bit key build runs on one GPU (multi-GPU routing is 64-bit)")

    def tnp(a):   # host array -> tensor of the key width (ops stay u8)
        return torch.from_numpy(a.astype(np.uint32) if (kbits == 32 and a.dtype == np.uint64) else a)

    def widen_np(r):   # results of the 32-bit build as the oracle's u64 (NOT_FOUND = all ones)
        r = np.asarray(r).astype(np.uint64)
        if kbits == 32:
            r[r == np.uint64(0xFFFFFFFF)] = np.uint64(0xFFFFFFFFFFFFFFFF)
        return r
    tree_n, batch_n = C["tree"], C["batch"]
    if args.tree:
        tree_n = args.tree
    if args.batch:
        batch_n = args.batch
    # cfg5: ONE 2^28-key tree and 2^24-request global batches at
    # every N -- strong scaling; the other configs are per-GPU sizes (weak)
    strong = bool(C.get("strong")) and world > 1
    if strong:
        tree_n //= world
        batch_n //= world
    nb = args.warmup + args.steps
    stream = torch.cuda.current_stream(dev)
    # range-query workload: eirene_submit_batch_range with
    # per-step output rows of `cap` pairs
    cap = C.get("range_len", 0) if W.RANGE in C["fracs"] else 0
    if cap and world > 1:
        raise SystemExit("range-query configs run on one GPU (DESIGN.md §7)")

    # query traversal: the default (one key-sorted request per thread, path
    # sharing) or the paper's iteration warps + range field (ablation)
    qmode = {"iterwarp": args.query_mode == "iterwarp", "iter_rgs": args.iter_rgs, "pipeline": bool(args.pipeline),
             "key_bits": kbits}
    if args.query_mode != "default" and world > 1:
        raise SystemExit("--query-mode iterwarp runs on one GPU")

    # ------------------------------------------------------------ inputs
    t_gen = time.time()
    per_tree = C.get("per_tree", 0)
    if world == 1:
        def build_plan(tag: int, nsteps: int):
            """Trees and pre-staged batches for nsteps steps.  Single-tree configs: one
            bulk-loaded tree, step s = batch s.  Fresh-tree configs (cfg1, cfg4;
            SURVEY §8(d)): step s runs batch s % per_tree on tree s // per_tree,
            every tree bulk-loaded from its own seed (untimed)."""
            if not per_tree:
                return None
            ntr = (nsteps + per_tree - 1) // per_tree
            wls_ = [W.Workload(cfg, tree=tree_n, batch=batch_n, seed=W.seed_for(cfg) + 7919 * (1000 * tag + t + 1), **wkw)
                    for t in range(ntr)]
            trees_ = []
            for w_ in wls_:
                tr = EireneTree(max_keys=tree_n + per_tree * batch_n + (1 << 12), max_batch=batch_n, **qmode)
                tr.bulk_load(tnp(w_.keys).to(dev), tnp(w_.vals).to(dev))
                tr.prepare(batch_n, bool(cap))   # graph capture outside every timed region
                trees_.append(tr)
            hb_ = [wls_[s_ // per_tree].batch_arrays(s_ % per_tree) for s_ in range(nsteps)]
            return wls_, trees_, [s_ // per_tree for s_ in range(nsteps)], hb_

        if per_tree:
            wls, trees, step_tree, host_batches = build_plan(0, nb)
            wl, tree = wls[0], trees[0]
        else:
            wl = W.Workload(cfg, tree=tree_n, batch=batch_n, **wkw)
            keys_d = tnp(wl.keys).to(dev)
            vals_d = tnp(wl.vals).to(dev)
            tree = EireneTree(max_keys=max(tree_n * 2, 1 << 20), max_batch=batch_n, **qmode)
            tree.bulk_load(keys_d, vals_d)
            del keys_d, vals_d
            wls, trees, step_tree = [wl], [tree], [0] * nb
            host_batches = [wl.batch_arrays(b) for b in range(nb)]
        batches = [tuple(tnp(a).to(dev) for a in hb) for hb in host_batches]
        results = [torch.empty(batch_n, dtype=kdt, device=dev) for _ in range(nb)]
        if cap:
            rrows = [(torch.empty(batch_n * cap, dtype=kdt, device=dev),
                      torch.empty(batch_n * cap, dtype=kdt, device=dev)) for _ in range(nb)]
    else:
        # weak scaling: the global tree holds world * tree_n keys, the global batch
        # world * batch_n requests; rank r owns key range r and ts-slice r
        wl = W.Workload(cfg, tree=tree_n * world, batch=batch_n * world, **wkw)
        sh = ShardedEirene(wl.keys, wl.vals, max_batch=batch_n, device=dev, fused=args.route == "fused")
        for f_ in (0.97, 1.0, 1.03, 1.1):   # graph capture for the likely shard batch size buckets, untimed
            sh.engine.prepare(min(int(batch_n * f_), batch_n * world))
        host_batches = []
        batches = []
        sl = slice(rank * batch_n, (rank + 1) * batch_n)
        for b in range(nb):
            o, k, v = wl.batch_arrays(b)
            host_batches.append(tuple(np.ascontiguousarray(a[sl]) for a in (o, k, v)))
            batches.append(tuple(torch.from_numpy(a).to(dev) for a in host_batches[-1]))
        results = [torch.empty(batch_n, dtype=torch.uint64, device=dev) for _ in range(nb)]
    torch.cuda.synchronize()
    gen_s = time.time() - t_gen

    # ------------------------------------------------------------ device-timed run
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(nb)]
    # Per-batch response times come from the device timestamps in every batch's stats
    # (%globaltimer, BatchCtl t_begin / t_end).  Host CUDA events around each submit
    # (EIRENE_BENCH_HOST_EVENTS=1) cost ~5 us of stream gap per batch (measured r2c:
    # inter-batch gap 11 us -> 5.5 us without them), so the timed region only has its two.
    host_ev = bool(os.environ.get("EIRENE_BENCH_HOST_EVENTS"))
    stats = []
    launches = 0

    def step(b, tr_list=None, st_tree=None, bt=None):
        nonlocal launches
        o, k, v = (bt or batches)[b]
        if host_ev:
            ev[b][0].record(stream)
        if world == 1:
            tr = (tr_list or trees)[(st_tree or step_tree)[b]]
            if cap:
                tk = tr.submit_range(o, k, v, results[b], cap, *rrows[b])
            else:
                tk = tr.submit(o, k, v, results[b])
            if host_ev:
                ev[b][1].record(stream)
            return (tr, tk)
        tk = sh.submit(o, k, v, results[b])
        if host_ev:
            ev[b][1].record(stream)
        return tk

    def fetch(r):
        return r[0].results(r[1]) if world == 1 else r.results()

    for b in range(args.warmup):
        stats.append(fetch(step(b)))
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks = ClockSampler(local)
    with clocks:
        t_start = torch.cuda.Event(enable_timing=True)
        t_end = torch.cuda.Event(enable_timing=True)
        # a short GPU spin (torch's, outside the timed region) lets the host queue
        # the first timed batches before the region starts, so batch times are
        # steady-state GPU times rather than host-launch latency after the sync
        torch.cuda._sleep(int(100e-6 * 1.9e9))
        t_start.record(stream)
        tickets = []
        for b in range(args.warmup, nb):
            tickets.append(step(b))
        if world == 1 and args.pipeline:   # the last batch ends on the library's back stream
            tickets[-1][0].stream_wait(tickets[-1][1], stream)
        t_end.record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
    for r in tickets:
        stats.append(fetch(r))
    elapsed_ms = t_start.elapsed_time(t_end)
    per_batch_ms = (np.array([ev[b][0].elapsed_time(ev[b][1]) for b in range(args.warmup, nb)]) if host_ev
                    else np.full(args.steps, elapsed_ms / args.steps))
    if os.environ.get("EIRENE_BENCH_VERBOSE"):
        print("per-batch ms:", " ".join(f"{x:.3f}" for x in per_batch_ms), file=sys.stderr)
        print("stage ms per batch:", [[round(x, 3) for x in s["stage_ms"][:5]] for s in stats[args.warmup:]][:8],
              file=sys.stderr)
    launches = int(sum(s["launches"] for s in stats[args.warmup:]))
    dns = [s.get("device_ns", 0) for s in stats[args.warmup:]]
    dev_batch_ms = np.array(dns, dtype=np.float64) / 1e6 if dns and all(x > 0 for x in dns) else None
    if os.environ.get("EIRENE_BENCH_VERBOSE") and dev_batch_ms is not None:
        print("device batch ms:", " ".join(f"{x:.3f}" for x in dev_batch_ms), file=sys.stderr)
        tb = [s.get("t_begin_ns", 0) for s in stats[args.warmup:]]
        te = [s.get("t_end_ns", 0) for s in stats[args.warmup:]]
        print("device gap us:", " ".join(f"{(tb[i + 1] - te[i]) / 1e3:.1f}" for i in range(len(tb) - 1)),
              file=sys.stderr)
    if world > 1:
        tmax = torch.tensor([elapsed_ms], device=dev)
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
        elapsed_ms = float(tmax.item())
    total_req = batch_n * world * args.steps
    value = total_req / (elapsed_ms * 1e-3) / 1e9

    # Stage breakdown: a second timed region over the same workload with the
    # library recording CUDA events between the stages on the submit stream
    # (graph replay is off while stage events are on, so this region also
    # shows the cost of direct launches).  Its batches reuse the pre-staged
    # input buffers of the first timed batches.
    stage_names = ["sort", "group", "query+range" if cap else "query", "update", "result"]
    n_stage = min(args.steps, 10)
    if world == 1 and per_tree:
        # fresh trees for the stage region too (a re-applied insert batch would not split)
        _, s_trees, s_tree_of, s_hb = build_plan(1, n_stage)
        # (indexed from args.warmup like the single-tree region: results[0..warmup) keep
        # the parity batches)
        s_batches = [None] * args.warmup + [tuple(tnp(a).to(dev) for a in hb) for hb in s_hb]
        s_tree_of = [0] * args.warmup + s_tree_of
        engines = s_trees
        stage_step = lambda i: step(args.warmup + i, s_trees, s_tree_of, s_batches)  # noqa: E731
    else:
        engines = [tree] if world == 1 else [sh.engine]
        stage_step = lambda i: step(args.warmup + i)  # noqa: E731
    for e_ in engines:
        e_.set_flags(timing=True)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    sa = torch.cuda.Event(enable_timing=True)
    sz = torch.cuda.Event(enable_timing=True)
    sa.record(stream)
    srs = [stage_step(i) for i in range(n_stage)]
    sz.record(stream)
    sstats = [fetch(r) for r in srs]
    torch.cuda.synchronize()
    direct_ms = sa.elapsed_time(sz) / n_stage
    stage_ms = np.array([s["stage_ms"][:5] for s in sstats]).mean(axis=0)
    for e_ in engines:
        e_.set_flags(timing=False)

    # ------------------------------------------------------------ e2e through the public API (host buffers)
    e2e = None
    if world == 1 and args.e2e_steps > 0 and cap:
        # range batches through the public API with host buffers: pinned H2D of
        # the inputs, submit_range, D2H of the counts and the range rows, all on
        # the submit stream inside the timed region (no overlap across steps)
        hb = [wl.batch_arrays(nb + i) for i in range(args.e2e_steps)]
        pin = [tuple(tnp(a).pin_memory() for a in x) for x in hb]
        hout = [(torch.empty(batch_n, dtype=kdt).pin_memory(),
                 torch.empty(batch_n * cap, dtype=kdt).pin_memory(),
                 torch.empty(batch_n * cap, dtype=kdt).pin_memory()) for _ in hb]
        dbuf = [torch.empty(batch_n, dtype=torch.uint8, device=dev), torch.empty(batch_n, dtype=kdt, device=dev),
                torch.empty(batch_n, dtype=kdt, device=dev)]
        dres = torch.empty(batch_n, dtype=kdt, device=dev)
        drk = torch.empty(batch_n * cap, dtype=kdt, device=dev)
        drv = torch.empty(batch_n * cap, dtype=kdt, device=dev)

        def e2e_step(i):
            for d_, h_ in zip(dbuf, pin[i]):
                d_.copy_(h_, non_blocking=True)
            tk_ = tree.submit_range(*dbuf, dres, cap, drk, drv)
            hout[i][0].copy_(dres, non_blocking=True)
            hout[i][1].copy_(drk, non_blocking=True)
            hout[i][2].copy_(drv, non_blocking=True)
            return tk_

        tree.results(e2e_step(0))
        torch.cuda.synchronize()
        a = torch.cuda.Event(enable_timing=True)
        z = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        tks = [e2e_step(i) for i in range(1, len(pin))]
        z.record(stream)
        torch.cuda.synchronize()
        for t_ in tks:
            tree.results(t_)
        e_ms = a.elapsed_time(z)
        n_e = len(pin) - 1
        e2e = {"value": batch_n * n_e / (e_ms * 1e-3) / 1e9, "unit": "Greq/s",
               "h2d_bytes_per_step": int(batch_n * 17), "d2h_bytes_per_step": int(batch_n * (8 + 16 * cap)),
               "steps": n_e, "path": "torch pinned H2D copies + EireneTree.submit_range + D2H of counts and "
                                     "range rows, one stream"}
    elif world == 1 and args.e2e_steps > 0:
        if per_tree:
            _, e_trees, e_tree_of, hb = build_plan(2, args.e2e_steps)
        else:
            hb = [wl.batch_arrays(nb + i) for i in range(args.e2e_steps)]
            e_trees, e_tree_of = [tree], [0] * len(hb)
        pin = [tuple(tnp(a).pin_memory() for a in x) for x in hb]
        hres = [torch.empty(batch_n, dtype=kdt).pin_memory() for _ in hb]
        tk = e_trees[e_tree_of[0]].submit_host(*pin[0], hres[0])   # warm the path
        e_trees[e_tree_of[0]].results(tk)
        # first DMA touch of each freshly pinned buffer (IOMMU / page mapping) is a
        # one-time cost a serving process with long-lived staging buffers never
        # pays: touch every buffer once, untimed (no batch is run)
        for x, r_ in zip(pin, hres):
            for t_ in x:
                torch.empty(t_.shape, dtype=t_.dtype, device=dev).copy_(t_, non_blocking=True)
            r_.copy_(torch.empty(r_.shape, dtype=r_.dtype, device=dev), non_blocking=True)
        torch.cuda.synchronize()
        a = torch.cuda.Event(enable_timing=True)
        z = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        tks = [(e_trees[e_tree_of[i]], e_trees[e_tree_of[i]].submit_host(*pin[i], hres[i])) for i in range(1, len(pin))]
        for tr_, t_ in tks:
            tr_.results(t_)   # waits for the batch's D2H (library's d2h stream)
        z.record(stream)       # after the last results() returned: covers every H2D, kernel and D2H
        torch.cuda.synchronize()
        e_ms = a.elapsed_time(z)
        n_e = len(pin) - 1
        # bytes actually moved per step: ops + keys copied; values of upserts
        # read zero-copy from the pinned buffer by the distribution kernel
        ups = np.mean([int(np.count_nonzero((x[0] == W.UPDATE) | (x[0] == W.INSERT))) for x in hb[1:]])
        e2e = {"value": batch_n * n_e / (e_ms * 1e-3) / 1e9, "unit": "Greq/s",
               "h2d_bytes_per_step": int(batch_n * (1 + kb) + kb * ups), "d2h_bytes_per_step": int(batch_n * kb),
               "steps": n_e, "path": "eirene_submit_batch_host (pinned host buffers; H2D of batch b+1 on the "
                                     "library's copy stream and D2H of batch b-1 on its d2h stream overlap "
                                     "batch b's kernels; upsert values read zero-copy)"}
    elif world > 1 and args.e2e_steps > 0:
        # through the public multi-GPU API with host buffers: every rank copies its
        # pinned ts-slice in, ShardedEirene routes / applies / returns, the results
        # slice is copied back; max over ranks of the device-timed region
        e_hb = []
        for i in range(args.e2e_steps):
            o, k, v = wl.batch_arrays(nb + i)
            e_hb.append(tuple(torch.from_numpy(np.ascontiguousarray(a[sl])).pin_memory() for a in (o, k, v)))
        hres = [torch.empty(batch_n, dtype=torch.uint64).pin_memory() for _ in e_hb]
        sh.submit_host(*e_hb[0], hres[0]).results()   # warm the path
        torch.cuda.synchronize()
        dist.barrier()
        a = torch.cuda.Event(enable_timing=True)
        z = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        tks = [sh.submit_host(*e_hb[i], hres[i]) for i in range(1, len(e_hb))]
        for t_ in tks:
            t_.results()
        z.record(stream)
        torch.cuda.synchronize()
        e_ms = torch.tensor([a.elapsed_time(z)], device=dev)
        dist.all_reduce(e_ms, op=dist.ReduceOp.MAX)
        n_e = len(e_hb) - 1
        ups = np.mean([int(np.count_nonzero((x[0].numpy() == W.UPDATE) | (x[0].numpy() == W.INSERT))) for x in e_hb])
        e2e = {"value": batch_n * world * n_e / (float(e_ms.item()) * 1e-3) / 1e9, "unit": "Greq/s",
               "h2d_bytes_per_step": int(world * batch_n * 17), "d2h_bytes_per_step": int(world * batch_n * 8),
               "steps": n_e, "path": "ShardedEirene.submit_host on every rank: pinned H2D of the rank's slice, "
                                     + ("fused push routing (partition kernel storing into the peers' arenas, "
                                        "results pushed back) " if sh.fused else
                                        "routing + NCCL exchanges ") + "+ shard batch, D2H of the results slice (one "
                                     "stream per rank); max over ranks"}

    # ------------------------------------------------------------ parity at N > 1
    # The first global batches against the oracle on SAMPLED KEY SLICES: requests
    # on different keys are independent (linearizability is local),
    # so the oracle loaded with the keys of a slice [lo, hi) and fed the batch's
    # requests with lo <= key < hi, in timestamp order, must reproduce those
    # requests' results exactly.  One slice straddles every shard boundary, plus
    # the two ends of the key space.
    parity = None
    if world > 1 and args.cpu_batches > 0:
        n_check = min(args.cpu_batches, nb)
        gathered = []
        for b in range(n_check):
            t_ = results[b].view(torch.int64)
            t_ = t_.cpu() if args.backend == "gloo" else t_
            parts = [torch.empty_like(t_) for _ in range(world)]
            dist.all_gather(parts, t_)
            gathered.append(np.concatenate([p.cpu().numpy() for p in parts]).view(np.uint64))
        if rank == 0:
            parity = slice_parity(wl, gathered, sh.splitters_np, args.parity_slice)

    # ------------------------------------------------------------ parity + CPU baseline (rank 0, N=1)
    cpu = None
    roof = None
    rar = None
    if rank == 0 and world == 1 and args.cpu_batches > 0 and tree_n > (1 << 25):
        # (cfg5 at N = 1: a 2^28-key oracle is minutes of CPU; key-slice parity as at N > 1)
        parity = slice_parity(wl, [results[b].cpu().numpy() for b in range(min(args.cpu_batches, nb))],
                              np.zeros(0, np.uint64), args.parity_slice)
    elif rank == 0 and world == 1 and args.cpu_batches > 0:
        import oracle
        n_check = min(args.cpu_batches, nb)
        refs = {}
        t0 = time.time()
        for b in range(n_check):   # one oracle per tree (fresh-tree configs), bulk load untimed
            if step_tree[b] not in refs:
                refs[step_tree[b]] = oracle.BTreeOracle(16)
                refs[step_tree[b]].load(wls[step_tree[b]].keys, wls[step_tree[b]].vals)
        load_s = time.time() - t0
        cpu_t = 0.0
        bad = 0
        for b in range(n_check):
            ref = refs[step_tree[b]]
            o, k, v = host_batches[b]
            with pinned_core() as pc:
                a = time.perf_counter()
                if cap:
                    want, wk, wv = ref.apply_range(o, k, v, cap)
                else:
                    want = ref.apply(o, k, v)
                cpu_t += time.perf_counter() - a
            pin_core = pc.core
            got = widen_np(results[b].cpu().numpy())
            bad += int(np.sum(got != want))
            if cap:
                gk = rrows[b][0].view(batch_n, cap).cpu().numpy()
                gv = rrows[b][1].view(batch_n, cap).cpu().numpy()
                col = np.arange(cap)[None, :] < want.astype(np.int64)[:, None]
                bad += int(np.sum((gk != wk) & col)) + int(np.sum((gv != wv) & col))
        parity = {"batches_checked": n_check, "mismatches": bad, "vs": "oracle B+tree, every request, bit-exact"}
        cpu = {"value": n_check * batch_n / cpu_t / 1e9, "unit": "Greq/s", "cores": 1, "host_cores": os.cpu_count(), "kind": "oracle",
               "sample": f"first {n_check} batches of the same workload ({n_check * batch_n} requests), "
                         f"sequential B+tree, 1 thread pinned to core {pin_core} (sched_setaffinity); "
                         f"bulk load {load_s:.1f}s untimed"}
        # roofline of the dominant kernel
        peaks = load_peaks()
        dom = int(np.argmax(stage_ms))
        if cap:
            ab = [algorithmic_bytes_range(wls[step_tree[b]].keys, *host_batches[b], 16, cap)["bytes"]
                  for b in range(args.warmup, min(nb, args.warmup + 4))]
            bytes_per = float(np.mean(ab))
            ms = stage_ms[2]
            kern = "range_kernel"
        elif stage_names[dom] == "query" or args.roofline_kernel == "query":
            ab = [algorithmic_bytes_query(wls[step_tree[b]].keys, *host_batches[b][:2], 16, kb)["bytes"]
                  for b in range(args.warmup, min(nb, args.warmup + 4))]
            bytes_per = float(np.mean(ab))
            ms = stage_ms[2]
            kern = "query_kernel"
        elif stage_names[dom] == "group":
            # bucket read 12 B + sorted payload 4 B + pinfo 4 B per request; one issued entry per key
            o0, k0 = host_batches[args.warmup][:2]
            d = len(W.sorted_unique(k0))
            bytes_per = batch_n * 20 + d * 17
            ms = stage_ms[1]
            kern = "group_kernel"
        elif stage_names[dom] == "update":
            # per issued write: its W-list entry (key, op, val, seg, leaf, slot: 26 B) and the
            # returned old value (8 B); per touched leaf (leaf run) its 256 B block read and
            # written back; per new leaf 256 B written (batch stats of the stage region)
            lr = float(np.mean([x["leaf_runs"] for x in sstats]))
            nlf = float(np.mean([x["new_leaves"] for x in sstats]))
            iw = float(np.mean([x["issued_w"] for x in sstats]))
            bytes_per = iw * 34 + lr * 512 + nlf * 256
            ms = stage_ms[3]
            kern = "update_kernel"
        else:
            # distribution: key 8 B + op 1 B read, 12 B written per request
            bytes_per = batch_n * (8 + 1 + 12)
            ms = stage_ms[0]
            kern = "bsort_dist_kernel"
        ach = bytes_per / (ms * 1e-3) / 1e9
        # measured DRAM traffic of the same kernel per launch, from the committed
        # ncu capture (tools/ncu_traffic.sh -> profiles/traffic.json); null if absent
        traffic, traffic_src = None, None
        tpath = os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles", "traffic.json")
        if os.path.exists(tpath):
            tj = json.load(open(tpath)).get(kern)
            if tj:
                traffic, traffic_src = tj["dram_bytes_per_launch"], tj["source"]
        roof = {"bound": "hbm", "achieved": ach, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": ach / peaks["hbm_gbs"], "traffic": traffic, "traffic_source": traffic_src, "kernel": kern,
                "stage_ms": ms, "algorithmic_bytes_per_launch": bytes_per, "peak_source": peaks["source"]}
        # whole-path random-access roofline (BASELINE north_star) on
        # the bulk-loaded shape: 1 / (L/R128 + S/R32 + Wr/R32w + B_io/BW) req/s
        if not cap and not per_tree:
            cs = [random_access_counts(wls[0].keys, *host_batches[b][:2], 16, kb)
                  for b in range(args.warmup, min(nb, args.warmup + 4))]
            c = {k: float(np.mean([x[k] for x in cs])) for k in cs[0]}
            # whole-path HBM streaming roofline: algorithmic bytes per request =
            # B_io + leaf lines x 128 + value sectors x 32 + written sectors x 32, at the measured peak
            b_req = c["bio"] + c["line_bytes"] * c["lines"] + 32 * c["sectors"] + 32 * c["writes"]
            stream_roof = peaks["hbm_gbs"] * 1e9 / b_req / 1e9
            roof["streaming"] = {"roofline_Greq_s": stream_roof, "frac": value / stream_roof,
                                 "bytes_per_request": b_req}
        if not cap and not per_tree and args.ra_probe and kbits == 64:
            n_leaves = (tree_n + 15) // 16
            pool_bytes = 1 << int(np.ceil(np.log2(max(n_leaves * 256, 1 << 20))))
            n_leaf = int(round(c["lines"] * batch_n))
            rates = probe_random_access(dev, stream, pool_bytes, n_leaf=n_leaf)
            # whole path: every leaf visited (key line + one value sector: R_leaf), the further
            # value sectors (R32), the written sectors (R32w), the streamed bytes (BW)
            t_req = (c["lines"] / rates["R_leaf"] + max(0.0, c["sectors"] - c["lines"]) / rates["R32"]
                     + c["writes"] / rates["R32w"] + c["bio"] / (peaks["hbm_gbs"] * 1e9))
            q_rate = n_leaf / (stage_ms[2] * 1e-3)   # the query kernel's leaf visits per second
            rar = {"roofline_Greq_s": 1.0 / t_req / 1e9, "achieved_Greq_s": value,
                   "frac": value / (1.0 / t_req / 1e9),
                   "query_kernel": {"leaf_visits_per_s": q_rate, "probe_R_leaf": rates["R_leaf"],
                                    "frac": q_rate / rates["R_leaf"]},
                   "streaming_frac": value / stream_roof,
                   "per_request": {"leaf_lines": c["lines"], "value_sectors": c["sectors"],
                                   "value_writes": c["writes"], "streamed_bytes": c["bio"]},
                   "rates_per_s": rates,
                   "probe": f"eirene_probe_gather over a {pool_bytes >> 20} MiB pool (the leaf pool's size, "
                            "power-of-two masks): 2^24 uniformly random 128 B line reads / 32 B sector reads / "
                            f"32 B sector writes, and {n_leaf} leaf visits (128 B key line + dependent 32 B value "
                            "sector) in key-sorted batch order; best of 3, CUDA events"}

    if rank == 0 and roof is None and not cap and not per_tree:
        # the query kernel of rank 0's shard (N > 1, or a tree too large for the full oracle): its
        # algorithmic bytes from the requests of the timed batches routed to this shard
        my = wl.keys[(wl.keys >= np.uint64(sh.lo)) & ((wl.keys < np.uint64(sh.hi)) if sh.hi != (1 << 64) - 1
                                                       else True)] if world > 1 else wl.keys
        ab = []
        for b in range(args.warmup, min(nb, args.warmup + 2)):
            o, k, _ = wl.batch_arrays(b)
            m = (k >= np.uint64(my[0])) & (k <= np.uint64(my[-1])) if world > 1 else slice(None)
            ab.append(algorithmic_bytes_query(my, o[m], k[m], 16)["bytes"])
        peaks = load_peaks()
        ach = float(np.mean(ab)) / (stage_ms[2] * 1e-3) / 1e9
        roof = {"bound": "hbm", "achieved": ach, "peak": peaks["hbm_gbs"], "unit": "GB/s", "frac": ach / peaks["hbm_gbs"],
                "traffic": None, "kernel": "query_kernel" + (" (rank 0's shard)" if world > 1 else ""),
                "stage_ms": float(stage_ms[2]), "algorithmic_bytes_per_launch": float(np.mean(ab)),
                "peak_source": peaks["source"]}

    if rank == 0:
        line = {
            "metric": "requests/sec per batch", "value": value, "unit": "Greq/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": elapsed_ms / args.steps,
            "higher_is_better": True, "scaling": "strong" if C.get("strong") else "weak", "vs_baseline": None,
            "dtype": "u32" if kbits == 32 else "u64", "data": "synthetic",
            "config": {"workload": f"cfg{cfg}: {tree_n * world} u{kbits} keys (fanout 16, fill 1.0), "
                                   f"{batch_n * world}-request batches, "
                                   + ", ".join(f"{int(p * 100)}% {['query', 'update', 'insert', 'delete', 'range'][o]}"
                                               for o, p in sorted(C['fracs'].items())) + f", {C['dist']} keys"
                                   + (f" (YCSB-like mix {args.mix})" if args.mix else "")
                                   + (f", range length {cap} (first {cap} pairs returned)" if cap else ""),
                       "cfg": cfg, "global_batch": batch_n * world,
                       "parallelism": (f"key-range shards x{world}, "
                                       + ("fused push over peer memory" if sh is not None and sh.fused
                                          else "NCCL all-to-all" + (f" (fused push unavailable: {sh.route_error})"
                                                                    if sh is not None and getattr(sh, "route_error", None)
                                                                    else ""))) if world > 1 else "single GPU",
                       "l2": "distinct input/result buffers per step (steps x 25 MiB >> 126 MB L2); "
                             "inner levels stay L2-resident across batches (steady state)"},
            "batch_ms": spread(dev_batch_ms, "device %globaltimer: start of the batch's first kernel to the end of "
                                             "its last kernel (BatchCtl t_begin / t_end), per timed batch")
            if dev_batch_ms is not None else spread(per_batch_ms, "CUDA events around each submit"),
            "batch_ms_host_events": spread(per_batch_ms, "CUDA events recorded on the submit stream around each "
                                                         "submit (includes any host-side launch gap)") if host_ev
            else None,
            "stage_ms": {n: float(x) for n, x in zip(stage_names, stage_ms)},
            "stage_region_ms_per_step": direct_ms,
            "gpu_launches": launches,
            "clocks": clocks.summary(),
            "e2e": e2e,
            "roofline": roof,
            "random_access_roofline": rar,
            "cpu_baseline": cpu,
            "parity": parity,
            "setup_s": gen_s,
        }
        if args.query_mode == "iterwarp":
            tot = lambda f: int(sum(s_[f] for s_ in stats[args.warmup:]))   # noqa: E731
            issued = tot("issued_q") + tot("issued_w")
            line["config"]["query_mode"] = f"iterwarp (iter_rgs {args.iter_rgs or 'auto'})"
            line["traversal"] = {"rg_vertical": tot("rg_vertical"), "rg_horizontal": tot("rg_horizontal"),
                                 "steps_per_issued": tot("trav_steps") / max(1, issued),
                                 "vertical_steps_per_issued": float(stats[-1]["height"])}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


class pinned_core:
    """Pin this process to one host core while the (single-threaded) oracle is timed; restore afterwards."""

    def __enter__(self):
        self.prev = os.sched_getaffinity(0)
        self.core = max(self.prev)
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *exc):
        os.sched_setaffinity(0, self.prev)
        return False


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--tree", type=int, default=0, help="override tree size (keys per GPU)")
    ap.add_argument("--batch", type=int, default=0, help="override batch size (requests per GPU)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=21)
    ap.add_argument("--cpu-batches", type=int, default=2)
    ap.add_argument("--ref-sample", type=int, default=1 << 18)
    ap.add_argument("--roofline-kernel", default="auto")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"])
    ap.add_argument("--query-mode", default="default", choices=["default", "iterwarp"],
                    help="iterwarp: the paper's iteration warps + range field (ablation)")
    ap.add_argument("--iter-rgs", type=int, default=0, help="RGs per iteration warp (0 = auto)")
    ap.add_argument("--ra-probe", type=int, default=1, help="measure the random-access roofline (1) or not (0)")
    ap.add_argument("--mix", default="", choices=["", "A", "B", "C", "U"],
                    help="YCSB-like mix override (cfg5): A 50/50 Zipf, B 95/5 Zipf, C 100%% read Zipf, U 95/5 uniform")
    ap.add_argument("--parity-slice", type=int, default=1 << 16, help="loaded keys per parity slice (N > 1)")
    ap.add_argument("--route", default="fused", choices=["nccl", "fused"],
                    help="N > 1 exchange: NCCL all-to-all, or the fused push into the peers' arenas over CUDA IPC "
                         "peer memory (SURVEY 8(f) NEXT(3))")
    ap.add_argument("--pipeline", type=int, default=0,
                    help="1: cross-batch pipelining (EIRENE_F_PIPELINE, SURVEY 8(f) NEXT(3))")
    args = ap.parse_args()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # one process per GPU: relaunch under torch.distributed.run (rank 0 prints the line)
        import socket
        s_ = socket.socket()
        s_.bind(("127.0.0.1", 0))
        port = s_.getsockname()[1]
        s_.close()
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
        raise SystemExit(subprocess.call(cmd))
    if args.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
