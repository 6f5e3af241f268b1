"""Where does C3's GPU idle time go?  Host wall time per call type vs GPU kernel
time, on the C3 TW stream at scale 0.25 (measurement only)."""
import os
import sys
import time
from collections import defaultdict

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_icde_lizlhs21_b200 import workload as W
from paper_conf_icde_lizlhs21_b200.table import Table

scale = float(os.environ.get("SCALE", "0.25"))
wl = W.c3_dynamic(scale=scale, shape="TW", batch=int(1_000_000 * min(1.0, scale * 4)), r=0.2, cycles=2)
dev = lambda a: torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).cuda()  # noqa
staged = [(b.op, dev(b.keys), dev(b.values) if b.values is not None else None) for b in wl.batches]
g = Table(d=4, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta, bucket_slots=8)
outs = {}
for op, k, v in staged:
    n = k.numel()
    if n not in outs:
        outs[n] = (torch.empty(n, dtype=torch.uint8, device="cuda"), torch.empty(n, dtype=torch.int32, device="cuda"))


def run(prealloc):
    g.clear()
    host = defaultdict(float)
    for op, k, v in staged:
        st, vo = outs[k.numel()]
        t0 = time.perf_counter()
        if op == "insert":
            g.insert(k, v, st) if prealloc else g.insert(k, v)
        elif op == "find":
            g.find(k, vo, st) if prealloc else g.find(k)
        else:
            g.delete(k, vo, st) if prealloc else g.delete(k)
        host[op] += time.perf_counter() - t0
    torch.cuda.synchronize()
    return host


for prealloc in (False, True, True):
    run(prealloc)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    g.profile(True)
    a.record()
    host = run(prealloc)
    b.record()
    torch.cuda.synchronize()
    prof = g.profile_read()
    g.profile(False)
    kern = sum(v[0] for v in prof.values())
    print(f"prealloc={prealloc} total {a.elapsed_time(b):.2f} ms, kernels {kern:.2f} ms, host per op type (ms):",
          {k: round(v * 1e3, 2) for k, v in host.items()}, "batches", len(staged), "stats", g.stats()["n_upsize"])
