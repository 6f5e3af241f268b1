"""Per-kernel times of the C2 step for several binning configurations (measurement only)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_icde_lizlhs21_b200 import workload as W
from paper_conf_icde_lizlhs21_b200.table import Table

log2n = int(os.environ.get("LOG2N", "27"))
cap, k, v, q, dk = W.c2_rand_static_torch(log2n, device="cuda")
n = 1 << log2n
confs = [tuple(int(x) for x in c.split(",")) for c in (sys.argv[1:] or ["1,0,0", "2,0,0"])]
st = torch.empty(n, dtype=torch.uint8, device="cuda")
vo = torch.empty(n, dtype=torch.int32, device="cuda")
fo = torch.empty(n, dtype=torch.uint8, device="cuda")
for c in confs:
    g = Table(d=4, init_capacity=cap, alpha=0.3, beta=0.85, bucket_slots=8, binning=c)
    res = {}
    for rep in range(3):
        g.clear()
        torch.cuda.synchronize()
        g.profile(True)
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        ev[0].record()
        g.insert(k, v, st)
        ev[1].record()
        g.find(q, vo, fo)
        ev[2].record()
        g.delete(dk, None, None)
        ev[3].record()
        torch.cuda.synchronize()
        prof = g.profile_read()
        g.profile(False)
    res["phase_ms"] = [round(ev[i].elapsed_time(ev[i + 1]), 3) for i in range(3)]
    res["kernels"] = {a: (round(b[0], 3), b[1]) for a, b in prof.items() if b[1]}
    res["binned"] = g.binning_info()
    print(json.dumps({"binning": c, **res}), flush=True)
    del g
    torch.cuda.empty_cache()
