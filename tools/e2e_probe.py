"""Diagnostic: where the host path (eirene_submit_batch_host) spends its time."""
import os, sys, time
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_zhangz0lzl23_b200 import workload as W
from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree

dev = torch.device("cuda", 0)
C = W.CONFIGS[2]
wl = W.Workload(2, tree=C["tree"], batch=C["batch"])
tree = EireneTree(max_keys=C["tree"] * 2, max_batch=C["batch"])
tree.bulk_load(torch.from_numpy(wl.keys).to(dev), torch.from_numpy(wl.vals).to(dev))
hb = [wl.batch_arrays(i) for i in range(12)]
pin = [tuple(torch.from_numpy(a).pin_memory() for a in x) for x in hb]
hres = [torch.empty(C["batch"], dtype=torch.uint64).pin_memory() for _ in hb]
import ctypes
cudart = ctypes.CDLL("libcudart.so") if False else None
for rep in range(2):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    tks = []
    per = []
    for i in range(len(pin)):
        a = time.perf_counter()
        tks.append(tree.submit_host(*pin[i], hres[i]))
        per.append(1e3 * (time.perf_counter() - a))
    print("per-call ms:", " ".join(f"{x:.2f}" for x in per))
    t1 = time.perf_counter()
    for t_ in tks:
        tree.results(t_)
    t2 = time.perf_counter()
    n = len(pin)
    print(f"rep {rep}: submit loop {1e3*(t1-t0)/n:.3f} ms/batch (host), total {1e3*(t2-t0)/n:.3f} ms/batch")
# device-buffer path for comparison, same batches pre-staged
dbat = [tuple(torch.from_numpy(a).to(dev) for a in x) for x in hb]
dres = [torch.empty(C["batch"], dtype=torch.uint64, device=dev) for _ in hb]
torch.cuda.synchronize()
t0 = time.perf_counter()
tks = [tree.submit(*dbat[i], dres[i]) for i in range(len(dbat))]
t1 = time.perf_counter()
for t_ in tks:
    tree.results(t_)
t2 = time.perf_counter()
print(f"device path: submit loop {1e3*(t1-t0)/len(dbat):.3f} ms/batch (host), total {1e3*(t2-t0)/len(dbat):.3f}")
# raw copies alone, same pattern: H2D 9 MB on s1, D2H 8 MB on s2
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
gk = torch.empty(C["batch"], dtype=torch.uint64, device=dev); go = torch.empty(C["batch"], dtype=torch.uint8, device=dev)
torch.cuda.synchronize(); t0 = time.perf_counter()
for i in range(len(pin)):
    with torch.cuda.stream(s1):
        gk.copy_(pin[i][1], non_blocking=True); go.copy_(pin[i][0], non_blocking=True)
    with torch.cuda.stream(s2):
        hres[i].copy_(dres[i], non_blocking=True)
torch.cuda.synchronize(); t2 = time.perf_counter()
print(f"raw copies only: {1e3*(t2-t0)/len(pin):.3f} ms/batch")
