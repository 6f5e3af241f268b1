"""Hash-partitioned DyCuckoo across the ranks of a torch.distributed group
(DESIGN.md §7).

Keys are owned by shard(k) = x_{d+1}(k) mod G (the (d+1)-th universal hash of
P:L271, independent of the pair and bucket hashes).  Every rank holds one full
DyCuckoo table (its own d subtables and [alpha, beta] resizing); since ops on
different keys never interact, the union of the shards has exactly the
single-table semantics.  A batch issued on any rank is routed:

    route_count (kernel)  ->  all_to_all(counts)  ->  route_scatter (kernel)
    ->  all_to_all(keys[, values])  ->  local batch on the owner (kernels)
    ->  all_to_all(replies)  ->  route_unpermute (kernel)

torch.distributed (NCCL over NVLink on GPUs, gloo in the CPU tests) is the
plumbing for the exchanges; every data-parallel step runs in libdyc.so.  The
per-rank table is any object with the Table interface (insert/find/delete/
route_*); the CPU tests inject a plain one to exercise this orchestration.
"""
from __future__ import annotations

from typing import List, Optional, Tuple


def _torch():
    import torch
    return torch


class DistTable:
    def __init__(self, shard, group=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.shard = shard

    # ------------------------------------------------------------ exchange
    def _splits(self, counts) -> Tuple[List[int], List[int]]:
        torch = _torch()
        recv = torch.empty_like(counts)
        self.dist.all_to_all_single(recv, counts, group=self.group)
        both = torch.stack([counts, recv]).cpu()
        return both[0].tolist(), both[1].tolist()

    def _a2a(self, x, send_splits, recv_splits):
        torch = _torch()
        out = torch.empty(sum(recv_splits), dtype=x.dtype, device=x.device)
        self.dist.all_to_all_single(out, x, recv_splits, send_splits, group=self.group)
        return out

    def _route(self, keys, values=None):
        counts = self.shard.route_count(keys, self.world)
        kout, vout, pos = self.shard.route_scatter(keys, values, self.world, counts)
        send, recv = self._splits(counts)
        rk = self._a2a(kout, send, recv)
        rv = self._a2a(vout, send, recv) if values is not None else None
        return rk, rv, pos, send, recv

    def _reply(self, pos, send, recv, vals=None, status=None):
        # replies travel back with the splits reversed
        bv = self._a2a(vals, recv, send) if vals is not None else None
        bs = self._a2a(status, recv, send) if status is not None else None
        return self.shard.route_unpermute(pos, bv, bs)

    # ------------------------------------------------------------ batches
    def insert(self, keys, values):
        """Returns per-op status (uint8) in request order."""
        rk, rv, pos, send, recv = self._route(keys, values)
        st = self.shard.insert(rk, rv)
        _, s = self._reply(pos, send, recv, status=st)
        return s

    def find(self, keys):
        """Returns (values int32-as-uint32, found uint8) in request order."""
        rk, _, pos, send, recv = self._route(keys)
        v, f = self.shard.find(rk)
        return self._reply(pos, send, recv, vals=v, status=f)

    def delete(self, keys):
        """Returns (old values, status) in request order."""
        rk, _, pos, send, recv = self._route(keys)
        v, s = self.shard.delete(rk)
        return self._reply(pos, send, recv, vals=v, status=s)

    def stats(self):
        return self.shard.stats()


# ---------------------------------------------------------------- bench (N > 1)
def bench_multi_gpu(args, rank, world, local, metric, ClockSampler, measured_peaks, run_oracle_sample):
    """Weak scaling: every rank issues one C2-shaped batch of its own keys (2^log2n
    inserts, 2^log2n finds at 50% hit, 2^(log2n-1) deletes) through the router;
    each shard receives ~1/G of every rank's ops.  Time = max over ranks."""
    import statistics
    import torch
    import torch.distributed as dist
    from . import workload as W
    from .table import Table

    n = 1 << args.log2n
    cap, k_ins, v_ins, k_find, k_del = W.c2_rand_static_torch(args.log2n, device="cuda", key_base=rank * n,
                                                              miss_base=rank * n)
    shard = Table(d=4, init_capacity=cap, alpha=0.3, beta=0.85, bucket_slots=args.bucket_slots)
    dt = DistTable(shard)
    stream = torch.cuda.current_stream()

    def step(evs=None):
        if evs: evs[0].record(stream)
        shard.clear()
        st = dt.insert(k_ins, v_ins)
        if evs: evs[1].record(stream)
        v, f = dt.find(k_find)
        if evs: evs[2].record(stream)
        dv, ds = dt.delete(k_del)
        if evs: evs[3].record(stream)
        return st, f, ds

    st, f, ds = step()
    torch.cuda.synchronize()
    ok = torch.tensor([int((st == 1).all().item()), int(f.sum().item()), int(ds.sum().item())],
                      dtype=torch.int64, device="cuda")
    dist.all_reduce(ok)
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    dist.barrier()
    recs = []
    shard.launch_count(reset=True)
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        dist.barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for _ in range(args.steps):
            evs = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            step(evs)
            recs.append(evs)
        b.record(stream)
        torch.cuda.synchronize()
        dist.barrier()
    ms = torch.tensor([a.elapsed_time(b) / args.steps], dtype=torch.float64, device="cuda")
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    ms_per_step = float(ms.item())
    n_ops = (n + n + n // 2) * world
    phases = {p: statistics.mean(r[i].elapsed_time(r[i + 1]) for r in recs)
              for i, p in enumerate(["insert", "find", "delete"])}
    if rank != 0:
        return None
    return {
        "metric": metric, "value": n_ops / (ms_per_step * 1e-3) / 1e6, "unit": "Mops/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": f"C2-shaped batch per rank (2^{args.log2n} inserts, 2^{args.log2n} finds 50% hit, "
                               f"2^{args.log2n - 1} deletes), hash-partitioned over {world} shards, "
                               "NCCL all-to-all routing", "d": 4, "alpha": 0.3, "beta": 0.85,
                   "bucket_slots": args.bucket_slots, "parallelism": f"shard{world}"},
        "phase_ms_rank0": phases,
        "check": {"all_inserted_ranks": int(ok[0].item()), "found_total": int(ok[1].item()),
                  "deleted_total": int(ok[2].item()), "expected_found": world * n // 2,
                  "expected_deleted": world * n // 2},
        "gpu_launches": shard.launch_count(),
        "clocks": clk.summary(),
        "roofline": None, "cpu_baseline": None, "e2e": None,
    }
