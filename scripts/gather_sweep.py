"""Random-gather ceiling sweep: L2 fetch granularity x bytes per random read."""
import ctypes as C, os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icde_lizlhs21_b200 import _lib as L
lib = L.load_library()
torch.cuda.init()
buf = torch.empty(1263225728, dtype=torch.uint8, device="cuda")
sink = torch.zeros(1, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream()
v = C.c_uint32()
L.check(lib.dyc_get_l2_fetch_granularity(C.byref(v)), "get"); print("default L2 fetch granularity", v.value)
res = []
for gran in (32, 64, 128):
    L.check(lib.dyc_set_l2_fetch_granularity(gran), "set")
    lib.dyc_get_l2_fetch_granularity(C.byref(v))
    for bpr in (32, 64, 128):
        nreads = (1 << 28) * 32 // bpr
        for _ in range(2):
            L.check(lib.dyc_bench_gather(buf.data_ptr(), buf.numel(), nreads, bpr, 3, sink.data_ptr(), s.cuda_stream), "g")
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); lib.dyc_bench_gather(buf.data_ptr(), buf.numel(), nreads, bpr, 5, sink.data_ptr(), s.cuda_stream); b.record()
        torch.cuda.synchronize(); ms = a.elapsed_time(b)
        r = dict(gran=gran, got=v.value, bytes_per_read=bpr, ms=ms, useful_gbs=nreads * bpr / ms / 1e6, greads_s=nreads / ms / 1e6)
        print(json.dumps(r)); res.append(r)
json.dump(res, open("gpurun_out/gather_sweep.json", "w"), indent=1)
