"""Experiment: does ordering a batch by the region of its first-choice bucket let
the 126 MB L2 absorb probe 1 and the write-backs?  (torch does the sort here;
only a measurement, not the product path.)"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_icde_lizlhs21_b200 import workload as W
from paper_conf_icde_lizlhs21_b200.table import Table

B = int(os.environ.get("B", "8"))
log2n = 27
n = 1 << log2n
cap, k, v, q, dk = W.c2_rand_static_torch(log2n, device="cuda")
g = Table(d=4, init_capacity=cap, alpha=0.3, beta=0.85, bucket_slots=B)
nb = g.stats()["buckets"]


def region_order(keys, region_bytes):
    x, pr = g.hash_probe(keys)
    x = x.to(torch.int64) & 0xFFFFFFFF
    t1 = pr[:, 0].to(torch.int64)
    nbt = torch.tensor(nb, device="cuda", dtype=torch.int64)
    b1 = torch.gather(x, 1, (t1 + 1).unsqueeze(1)).squeeze(1) % nbt[t1]
    base = torch.cumsum(torch.cat([torch.zeros(1, device="cuda", dtype=torch.int64), nbt[:-1]]), 0)
    addr = (base[t1] + b1) * (8 * B)
    reg = addr // region_bytes
    return torch.argsort(reg, stable=True)


def timed(fn, reps=3):
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return min(ts)


res = {}
st = torch.empty(n, dtype=torch.uint8, device="cuda")


def ins(kk, vv):
    g.clear()
    g.insert(kk, vv, st)


res["insert_orig_ms"] = timed(lambda: ins(k, v))
for rb_mb in (8, 16, 32, 64, 128, 1 << 20):
    o = region_order(k, rb_mb << 20)
    ko, vo = k[o].contiguous(), v[o].contiguous()
    res[f"insert_sorted_{rb_mb}MB_ms"] = timed(lambda: ins(ko, vo))
g.clear()
g.insert(k, v, st)
vo_ = torch.empty(n, dtype=torch.int32, device="cuda")
fo_ = torch.empty(n, dtype=torch.uint8, device="cuda")
res["find_orig_ms"] = timed(lambda: g.find(q, vo_, fo_))
for rb_mb in (16, 32, 64):
    o = region_order(q, rb_mb << 20)
    qo = q[o].contiguous()
    res[f"find_sorted_{rb_mb}MB_ms"] = timed(lambda: g.find(qo, vo_, fo_))
g.profile(True)
g.find(q, vo_, fo_)
print(json.dumps(res, indent=1))
