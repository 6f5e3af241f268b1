"""C5 fill at N=1 with per-batch tracing: host ms of each insert call, GPU ms
(CUDA events), upsizes and cudaMalloc ms inside the call.  Explains where the
fill's time outside kernels goes (profiles/r1t_c5_variance.md)."""
import json
import sys
import time

import torch

sys.path.insert(0, ".")
from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import Table  # noqa: E402

torch.cuda.set_device(0)
log2k = 31
batch = 1 << 24
t = Table(d=4, init_capacity=1 << 20, alpha=0.3, beta=0.85, bucket_slots=8)
gen = W.c5_batches_torch(0, 1, device="cuda", log2_keys=log2k, batch=batch, mixed_batches=0)
fill = [item for item in gen if item[0] == "insert"]
torch.cuda.synchronize()
rows = []
s0 = t.stats()
t_all = time.perf_counter()
for i, (_, k, v) in enumerate(fill):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    st0 = t.stats()
    t.profile(True)
    torch.cuda.synchronize()
    h0 = time.perf_counter()
    e0.record()
    t.insert(k, v)
    e1.record()
    h1 = time.perf_counter()
    torch.cuda.synchronize()
    prof = t.profile_read()
    t.profile(False)
    st1 = t.stats()
    rows.append({"kernels": {k: (round(v[0], 2), v[1]) for k, v in prof.items() if v[1]},
                 "retries": st1["n_place_retry"] - st0["n_place_retry"],
                 "fail_upsizes": st1["n_fail_upsize"] - st0["n_fail_upsize"],
                 "evict": st1["n_evict"] - st0["n_evict"],"i": i, "host_ms": (h1 - h0) * 1e3, "gpu_ms": e0.elapsed_time(e1),
                 "upsizes": st1["n_upsize"] - st0["n_upsize"], "alloc_ms": st1["alloc_ms"] - st0["alloc_ms"],
                 "sync_ms": st1["sync_ms"] - st0["sync_ms"], "n_sync": st1["n_sync"] - st0["n_sync"],
                 "n_alloc": st1["n_device_alloc"] - st0["n_device_alloc"], "fill": st1["fill"]})
total = (time.perf_counter() - t_all) * 1e3
slow = sorted(rows, key=lambda r: -r["gpu_ms"])[:12]
print(json.dumps({"total_ms_incl_stats": total, "sum_gpu_ms": sum(r["gpu_ms"] for r in rows),
                  "sum_alloc_ms": sum(r["alloc_ms"] for r in rows), "slowest": slow}, indent=1))
