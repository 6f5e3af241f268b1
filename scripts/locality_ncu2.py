"""ncu companion of scripts/locality2.py: one C2 insert (then find) with the batch
in request order (MODE=orig) or ordered by first-choice region (MODE=sorted,
REGION_MB).  Run under ncu -k regex:'k_upsert|k_find|k_delete'."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_icde_lizlhs21_b200 import workload as W
from paper_conf_icde_lizlhs21_b200.table import Table

mode = os.environ.get("MODE", "orig")
rb = int(os.environ.get("REGION_MB", "64")) << 20
n = 1 << 27
cap, k, v, q, dk = W.c2_rand_static_torch(27, device="cuda")
g = Table(d=4, init_capacity=cap, alpha=0.3, beta=0.85, bucket_slots=8)
nb = g.stats()["buckets"]


def order(keys):
    x, pr = g.hash_probe(keys)
    x = x.to(torch.int64) & 0xFFFFFFFF
    t1 = pr[:, 0].to(torch.int64)
    nbt = torch.tensor(nb, device="cuda", dtype=torch.int64)
    b1 = torch.gather(x, 1, (t1 + 1).unsqueeze(1)).squeeze(1) % nbt[t1]
    base = torch.cumsum(torch.cat([torch.zeros(1, device="cuda", dtype=torch.int64), nbt[:-1]]), 0)
    return torch.argsort(((base[t1] + b1) * 64) // rb, stable=True)


if mode == "sorted":
    o = order(k)
    k, v = k[o].contiguous(), v[o].contiguous()
    q = q[order(q)].contiguous()
    dk = dk[order(dk)].contiguous()
torch.cuda.synchronize()
g.insert(k, v)
g.find(q)
g.delete(dk)
torch.cuda.synchronize()
print("done", mode)
