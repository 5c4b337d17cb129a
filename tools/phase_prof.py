"""Phase times of the distribution (bsort_dist_kernel) and group kernels from a
-DEIRENE_PHASE_PROF build (diagnostic):

    python -m paper_conf_ppopp_zhangz0lzl23_b200.build --variant phase -DEIRENE_PHASE_PROF
    EIRENE_LIB=paper_conf_ppopp_zhangz0lzl23_b200/libeirene_phase.so python tools/phase_prof.py [cfg]

Runs a few batches of the config, then prints, per phase, the median / max over
CTAs of the time since the kernel's earliest CTA start (us)."""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_zhangz0lzl23_b200 import _ffi, workload as W  # noqa: E402
from paper_conf_ppopp_zhangz0lzl23_b200.tree import EireneTree  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
C = W.CONFIGS[cfg]
dev = torch.device("cuda", 0)
wl = W.Workload(cfg, tree=C["tree"], batch=C["batch"])
t = EireneTree(max_keys=max(2 * C["tree"], 1 << 20), max_batch=C["batch"])
t.bulk_load(torch.from_numpy(wl.keys).to(dev), torch.from_numpy(wl.vals).to(dev))
names = {0: ["start", "hist", "bcount atomics", "barrier", "cut", "tile hist+cursor", "scatter"],
         1: ["ticket", "sort", "sweep1", "lookback", "emit", "ss:loaded+range", "ss:scan", "ss:rank"]}
acc = {0: [], 1: []}
for b in range(6):
    o, k, v = (torch.from_numpy(x).to(dev) for x in wl.batch_arrays(b))
    res = torch.empty(o.numel(), dtype=torch.uint64, device=dev)
    t.results(t.submit(o, k, v, res))
    buf = np.zeros(2 * 512 * 8, np.uint64)
    _ffi.check(_ffi.lib().eirene_debug_phases(t._h, buf.ctypes.data_as(ctypes.c_void_p), buf.size), "phases")
    if b < 2:
        continue
    p = buf.reshape(2, 512, 8).astype(np.int64)
    for kk in (0, 1):
        q = p[kk]
        q = q[q[:, 0] > 0]
        acc[kk].append(q - q[:, :1].min())
for kk in (0, 1):
    q = np.concatenate(acc[kk])
    print(["bsort_dist_kernel", "group_kernel"][kk], f"({q.shape[0] // 4} CTAs x 4 batches)")
    for i, nm in enumerate(names[kk]):
        col = q[:, i] / 1e3
        print(f"  {i} {nm:18s} median {np.median(col):7.2f} us   p90 {np.percentile(col, 90):7.2f}   max {col.max():7.2f}")
