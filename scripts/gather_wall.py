"""Where the random-access wall sits: dyc_bench_gather and
dyc_bench_gather_ex (read, then an 8-B store / 8-B CAS / 32-B sector store into
the bucket just read, address from the group's own probe only) at
an L2-resident and an HBM-sized buffer, 64-B buckets (2 lanes), timed with CUDA
events; run under ncu for the DRAM / L2 counters (scripts/gpu_pass.sh gather)."""
import ctypes as C
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_lizlhs21_b200 import _lib as L  # noqa: E402

lib = L.load_library()
sink = torch.zeros(1, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream()
reps = int(os.environ.get("GATHER_REPS", "3"))
out = []
for label, nbytes in (("l2_48MB", 48 << 20), ("hbm_1.26GB", 1263225728), ("hbm_8GB", 8 << 30)):
    buf = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    buf.fill_(7)
    for flags in (0, 1, 2, 4):   # read only, + 8-B store, + 8-B CAS, + 32-B sector store
        for bpr in (32, 64, 128):
            nreads = 1 << 27
            best = None
            for _ in range(reps):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                L.check(lib.dyc_bench_gather_ex(buf.data_ptr(), nbytes, nreads, bpr, 11, flags, sink.data_ptr(),
                                                 s.cuda_stream), "gather")
                b.record()
                torch.cuda.synchronize()
                ms = a.elapsed_time(b)
                best = ms if best is None else min(best, ms)
            r = dict(buffer=label, write={0: None, 1: 'store8', 2: 'cas8', 4: 'sector32'}[flags], bytes_per_read=bpr, ms=best, gops=nreads / best / 1e6,
                     useful_gbs=nreads * bpr / best / 1e6)
            print(json.dumps(r), flush=True)
            out.append(r)
    del buf
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/gather_wall.json", "w"), indent=1)
