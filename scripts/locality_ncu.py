import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icde_lizlhs21_b200 import workload as W
from paper_conf_icde_lizlhs21_b200.table import Table
exec(open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "locality_experiment.py")).read().split("res = {}")[0].split("B = int")[0])
B = 8
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
    return torch.argsort(((base[t1] + b1) * (8 * B)) // region_bytes, stable=True)
st = torch.empty(n, dtype=torch.uint8, device="cuda")
o = region_order(k, 64 << 20)
ko, vo = k[o].contiguous(), v[o].contiguous()
g.clear(); g.insert(k, v, st)     # unsorted
g.clear(); g.insert(ko, vo, st)   # sorted
torch.cuda.synchronize()
