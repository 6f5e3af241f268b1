"""Per-pass times of the staged path on C2 (2^LOG2N ops): profile scopes of the
library and, under `ncu --metrics gpu__time_duration.sum`, the launch list."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_icde_lizlhs21_b200 import workload as W
from paper_conf_icde_lizlhs21_b200.table import Table

log2n = int(os.environ.get("LOG2N", "27"))
mode = os.environ.get("STAGED", "force")
reps = int(os.environ.get("REPS", "2"))
n = 1 << log2n
cap, k, v, q, dk = W.c2_rand_static_torch(log2n, device="cuda")
g = Table(d=4, init_capacity=cap, alpha=0.3, beta=0.85, bucket_slots=8, staged=mode)
out = {}
for r in range(reps):
    g.clear()
    torch.cuda.synchronize()
    g.profile(True)
    g.profile_read()
    res = {}
    prev = {}
    for name, fn in (("insert", lambda: g.insert(k, v)), ("find", lambda: g.find(q)), ("delete", lambda: g.delete(dk))):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        res[name + "_ms"] = round(a.elapsed_time(b), 3)
        cur = {kk: vv[0] for kk, vv in g.profile_read().items() if vv[1]}
        res[name + "_kernels"] = {kk: round(vv - prev.get(kk, 0.0), 3) for kk, vv in cur.items() if vv - prev.get(kk, 0.0) > 0}
        prev = cur
    g.profile(False)
    out[f"rep{r}"] = res
out["stats"] = {kk: vv for kk, vv in g.stats().items() if kk in ("n_staged", "m", "n_sync")}
print(json.dumps(out, indent=1))
