"""Random bucket-read rate vs. buffer size (L2-resident vs HBM)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icde_lizlhs21_b200 import _lib as L
lib = L.load_library()
buf = torch.empty(1 << 31, dtype=torch.uint8, device="cuda")
sink = torch.zeros(1, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream()
out = []
for mb in (2, 8, 32, 64, 96, 128, 256, 1024, 2048):
    for bpr in (32, 64, 128):
        nreads = 1 << 27
        for _ in range(2):
            lib.dyc_bench_gather(buf.data_ptr(), mb << 20, nreads, bpr, 3, sink.data_ptr(), s.cuda_stream)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); lib.dyc_bench_gather(buf.data_ptr(), mb << 20, nreads, bpr, 5, sink.data_ptr(), s.cuda_stream); b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b)
        r = dict(buf_mb=mb, bytes=bpr, g_reads_s=round(nreads / ms / 1e6, 1), lanes=bpr // 32)
        print(json.dumps(r)); out.append(r)
json.dump(out, open("gpurun_out/l2_rate.json", "w"), indent=1)
