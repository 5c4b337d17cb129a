"""A/B timing of tuning variants on one tree (diagnostic, not a bench number).

    python tools/ab.py --config 2 --reps 4 --steps 30 "EIRENE_QCAP=8" "EIRENE_QCAP=16"

Each variant is a set of environment assignments read by the library at launch
time; variants run interleaved (rep-major) on the same tree so drift and clock
changes hit all of them alike; the median ms/batch per variant is printed.
"""
import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--reps", type=int, default=4)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--timing", action="store_true", help="also report per-stage ms (direct launches)")
    ap.add_argument("variants", nargs="+")
    a = ap.parse_args()
    import torch

    from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W
    from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree

    dev = torch.device("cuda", 0)
    C = W.CONFIGS[a.config]
    wl = W.Workload(a.config, tree=C["tree"], batch=C["batch"])
    tree = EireneTree(max_keys=max(C["tree"] * 2, 1 << 20), max_batch=C["batch"])
    tree.bulk_load(torch.from_numpy(wl.keys).to(dev), torch.from_numpy(wl.vals).to(dev))
    nb = a.steps + 3
    batches = [tuple(torch.from_numpy(x).to(dev) for x in wl.batch_arrays(b)) for b in range(nb)]
    res = torch.empty(C["batch"], dtype=torch.uint64, device=dev)
    stream = torch.cuda.current_stream(dev)
    out = {v: [] for v in a.variants}
    stages = {v: [] for v in a.variants}
    for rep in range(a.reps):
        for v in a.variants:
            for kv in v.split(","):
                k, _, x = kv.partition("=")
                if k:
                    os.environ[k] = x
            tree.set_flags(timing=False)   # drops cached graphs: launch configs are re-read
            for b in range(3):
                tree.submit(*batches[b], res)
            torch.cuda.synchronize()
            torch.cuda._sleep(int(100e-6 * 1.9e9))
            s0 = torch.cuda.Event(enable_timing=True)
            s1 = torch.cuda.Event(enable_timing=True)
            s0.record(stream)
            for b in range(3, nb):
                tree.submit(*batches[b], res)
            s1.record(stream)
            torch.cuda.synchronize()
            out[v].append(s0.elapsed_time(s1) / a.steps)
            if a.timing:
                tree.set_flags(timing=True)
                tks = [tree.submit(*batches[3 + b % a.steps], res) for b in range(8)]
                st = np.array([tree.results(t)["stage_ms"][:5] for t in tks]).mean(axis=0)
                stages[v].append(st)
            for kv in v.split(","):
                k, _, x = kv.partition("=")
                if k:
                    os.environ.pop(k, None)
        print(f"rep {rep}: " + "  ".join(f"{v}: {out[v][-1] * 1e3:.1f}us" for v in a.variants), flush=True)
    for v in a.variants:
        line = f"{v:40s} median {np.median(out[v]) * 1e3:7.1f} us/batch  min {min(out[v]) * 1e3:7.1f}"
        if a.timing:
            st = np.median(np.array(stages[v]), axis=0) * 1e3
            line += "  stages " + " ".join(f"{x:.1f}" for x in st)
        print(line)


if __name__ == "__main__":
    main()
