import os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W
from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree
dev = torch.device("cuda", 0)
w = W.Workload(2, tree=1 << 22, batch=1 << 20)
t = EireneTree(max_keys=1 << 23, max_batch=1 << 20, timing=True)
t.bulk_load(torch.from_numpy(w.keys).to(dev), torch.from_numpy(w.vals).to(dev))
for b in range(4):
    ops, keys, vals = w.batch_arrays(b)
    res, st = t.apply(torch.from_numpy(ops).to(dev), torch.from_numpy(keys).to(dev), torch.from_numpy(vals).to(dev))
    print({k: st[k] for k in ("issued_q", "issued_w", "leaf_runs", "retries", "stm_fallbacks", "leaf_splits")}, [round(x, 4) for x in st["stage_ms"][:6]], flush=True)
