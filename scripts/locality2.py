"""Experiment (round 2): with FUSE/FFI in the probe kernels, how much do insert,
find and delete gain when a C2 batch is ordered by the region of its
first-choice bucket?  torch does the ordering here (measurement only, not the
product path); per-kernel times come from the library's profiled scopes."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_icde_lizlhs21_b200 import workload as W
from paper_conf_icde_lizlhs21_b200.table import Table

log2n = int(os.environ.get("LOG2N", "27"))
n = 1 << log2n
cap, k, v, q, dk = W.c2_rand_static_torch(log2n, device="cuda")
g = Table(d=4, init_capacity=cap, alpha=0.3, beta=0.85, bucket_slots=8)
nb = g.stats()["buckets"]


def region_order(keys, region_bytes):
    x, pr = g.hash_probe(keys)
    x = x.to(torch.int64) & 0xFFFFFFFF
    t1 = pr[:, 0].to(torch.int64)
    nbt = torch.tensor(nb, device="cuda", dtype=torch.int64)
    b1 = torch.gather(x, 1, (t1 + 1).unsqueeze(1)).squeeze(1) % nbt[t1]
    base = torch.cumsum(torch.cat([torch.zeros(1, device="cuda", dtype=torch.int64), nbt[:-1]]), 0)
    addr = (base[t1] + b1) * 64
    return torch.argsort(addr // region_bytes, stable=True)


def timed(fn, setup=None, reps=3):
    ts, prof = [], None
    for _ in range(reps):
        if setup:
            setup()
        g.profile(True)
        g.profile_read()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        t = a.elapsed_time(b)
        p = {kk: round(vv[0], 3) for kk, vv in g.profile_read().items() if vv[1]}
        g.profile(False)
        if not ts or t < min(ts):
            prof = p
        ts.append(t)
    return round(min(ts), 3), prof


res = {}
st = torch.empty(n, dtype=torch.uint8, device="cuda")
vo_ = torch.empty(n, dtype=torch.int32, device="cuda")
fo_ = torch.empty(n, dtype=torch.uint8, device="cuda")


def fill(kk, vv):
    g.clear()
    g.insert(kk, vv, st)


res["insert_orig"] = timed(lambda: fill(k, v))
for rb_mb in (16, 32, 64):
    o = region_order(k, rb_mb << 20)
    ko, vo = k[o].contiguous(), v[o].contiguous()
    res[f"insert_sorted_{rb_mb}MB"] = timed(lambda: fill(ko, vo))
fill(k, v)
res["find_orig"] = timed(lambda: g.find(q, vo_, fo_))
for rb_mb in (16, 32, 64):
    o = region_order(q, rb_mb << 20)
    qo = q[o].contiguous()
    res[f"find_sorted_{rb_mb}MB"] = timed(lambda: g.find(qo, vo_, fo_))
res["delete_orig"] = timed(lambda: g.delete(dk, vo_[:dk.numel()], st[:dk.numel()]), setup=lambda: fill(k, v))
for rb_mb in (16, 32, 64):
    o = region_order(dk, rb_mb << 20)
    dko = dk[o].contiguous()
    res[f"delete_sorted_{rb_mb}MB"] = timed(lambda: g.delete(dko, vo_[:dk.numel()], st[:dk.numel()]),
                                            setup=lambda: fill(k, v))
# cost of the ordering itself with torch (argsort), for scale
res["torch_argsort_ms"] = timed(lambda: region_order(k, 32 << 20))[0]
print(json.dumps(res, indent=1))
