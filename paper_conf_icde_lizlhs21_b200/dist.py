"""Hash-partitioned DyCuckoo across the ranks of a torch.distributed group
(DESIGN.md §7): the Python-orchestrated routers and the
multi-GPU bench drivers.

The product path for sharding is the C ABI (dyc_dist_*, sharded.py), where
the routing and the NCCL exchange run inside libdyc.so.  This module keeps:

- DistTable: the same routing orchestrated from Python over
  torch.distributed all-to-all (the round-1 path, the baseline the C ABI
  replaced; its CPU orchestration tests run over gloo), and
- PeerRouter (DistTable(p2p=True)): fused dispatch/combine kernels that store
  straight into peer memory (CUDA IPC), with host barriers between phases,
- bench_multi_gpu / bench_c5: the bench's N > 1 and C5 drivers (C ABI by
  default, the fused peer path with --p2p).

Keys are owned by shard(k) = x_{d+1}(k) mod G (the (d+1)-th universal hash of
P:L271, independent of the pair and bucket hashes).  Every rank holds one full
DyCuckoo table (its own d subtables and [alpha, beta] resizing); since ops on
different keys never interact, the union of the shards has exactly the
single-table semantics.  DistTable routes a batch as

    route_count (kernel)  ->  all_to_all(counts)  ->  route_scatter (kernel)
    ->  all_to_all(keys[, values])  ->  local batch on the owner (kernels)
    ->  all_to_all(replies)  ->  route_unpermute (kernel)
"""
from __future__ import annotations

from typing import List, Optional, Tuple


def _torch():
    import torch
    return torch


class DistTable:
    """Routes single-type batches to the owning shards.  The batch is split into
    `chunks` pieces that are pipelined: the all-to-all of chunk c+1 (NCCL stream)
    runs while the owner executes chunk c (compute stream), and the replies of
    chunk c travel back while chunk c+1 executes.  Each rank must use the same
    `chunks` (collectives are issued in the same order everywhere)."""

    def __init__(self, shard, group=None, force_route: bool = False, chunks: int = 4, p2p: bool = False,
                 max_ops: Optional[int] = None, p2p_buffers=None, p2p_sync=None):
        import torch.distributed as dist
        self.force_route = force_route
        self.dist = dist
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.shard = shard
        self.chunks = max(1, int(chunks))
        self.last_recv = 0
        self.p2p = None
        if p2p:
            if not max_ops:
                raise ValueError("p2p routing needs max_ops (the largest batch any rank issues)")
            self.p2p = PeerRouter(self, int(max_ops), buffer_factory=p2p_buffers, sync=p2p_sync)

    # ------------------------------------------------------------ exchange
    def _a2a(self, x, send_splits, recv_splits, async_op=False):
        torch = _torch()
        out = torch.empty(sum(recv_splits), dtype=x.dtype, device=x.device)
        w = self.dist.all_to_all_single(out, x, recv_splits, send_splits, group=self.group, async_op=async_op)
        return out, w

    def _run(self, op, keys, values=None, n_out=1, begin=None, end=None, tags=None):
        if self.p2p is not None:
            return self.p2p.run(op, keys, values, n_out, begin, end, tags)
        return self._run_a2a(op, keys, values, n_out, begin, end, tags)

    def _run_a2a(self, op, keys, values=None, n_out=1, begin=None, end=None, tags=None):
        """Pipelined route -> all-to-all -> owner op -> all-to-all back -> unpermute.
        op(keys, values) returns a tuple of n_out per-op result tensors.  begin(n)
        / end() bracket the owner's parts so that they form ONE batch (one
        resize decision, one alpha check: dyc_*_begin/_part/_end)."""
        torch = _torch()
        n = keys.numel()
        C, W = self.chunks, self.world
        bounds = [n * c // C for c in range(C + 1)]
        parts, counts = [], []
        for c in range(C):
            kc = keys[bounds[c]:bounds[c + 1]]
            vc = values[bounds[c]:bounds[c + 1]] if values is not None else None
            cnt = self.shard.route_count(kc, W)
            if tags is None:
                kout, vout, pos = self.shard.route_scatter(kc, vc, W, cnt)
                tout = None
            else:
                kout, vout, pos, tout = self.shard.route_scatter(kc, vc, W, cnt, tags=tags[bounds[c]:bounds[c + 1]])
            parts.append((kout, vout, pos, tout))
            counts.append(cnt)
        # one exchange of every chunk's per-destination counts (row w: counts for rank w)
        send = torch.stack(counts).t().contiguous()
        recv = torch.empty_like(send)
        self.dist.all_to_all_single(recv, send, group=self.group)
        both = torch.stack([send, recv]).cpu()
        ssp = [both[0][:, c].tolist() for c in range(C)]
        rsp = [both[1][:, c].tolist() for c in range(C)]
        self.last_recv = int(both[1].sum())
        if begin is not None:
            begin(self.last_recv)
        fwd = []
        for c in range(C):
            kout, vout, _, tout = parts[c]
            rk, wk = self._a2a(kout, ssp[c], rsp[c], async_op=True)
            rv, wv = self._a2a(vout, ssp[c], rsp[c], async_op=True) if values is not None else (None, None)
            rt, wt = self._a2a(tout, ssp[c], rsp[c], async_op=True) if tags is not None else (None, None)
            fwd.append((rk, wk, rv, wv, rt, wt))
        back = []
        for c in range(C):
            rk, wk, rv, wv, rt, wt = fwd[c]
            for w_ in (wk, wv, wt):
                if w_ is not None:
                    w_.wait()
            res = op(rk, rv) if tags is None else op(rk, rv, rt)
            res = res if isinstance(res, tuple) else (res,)
            back.append([self._a2a(r, rsp[c], ssp[c], async_op=True) for r in res])
        if end is not None:
            end()
        # results land directly in their slice of the batch result (request order)
        out_s = torch.empty(n, dtype=torch.uint8, device=keys.device)
        out_v = torch.empty(n, dtype=torch.int32, device=keys.device) if n_out == 2 else None
        for c in range(C):
            for (r, w) in back[c]:
                w.wait()
            pos = parts[c][2]
            got = [r for (r, _) in back[c]]
            lo, hi = bounds[c], bounds[c + 1]
            if hi == lo:
                continue
            if n_out == 1:
                self.shard.route_unpermute(pos, None, got[0], out_status=out_s[lo:hi])
            else:
                self.shard.route_unpermute(pos, got[0], got[1], out_vals=out_v[lo:hi], out_status=out_s[lo:hi])
        return out_s if n_out == 1 else (out_v, out_s)

    # ------------------------------------------------------------ batches
    # With one rank there is nothing to exchange: the batch goes straight to the
    # local table (no collective is invented for a path that does not shard).
    def insert(self, keys, values):
        """Returns per-op status (uint8) in request order."""
        if self.world == 1 and not self.force_route:
            self.last_recv = keys.numel()
            return self.shard.insert(keys, values)
        return self._run(lambda k, v: self.shard.insert_part(k, v), keys, values, n_out=1,
                         begin=self.shard.insert_begin, end=self.shard.insert_end)

    def find(self, keys):
        """Returns (values int32-as-uint32, found uint8) in request order."""
        if self.world == 1 and not self.force_route:
            self.last_recv = keys.numel()
            return self.shard.find(keys)
        return self._run(lambda k, v: self.shard.find(k), keys, None, n_out=2)

    def delete(self, keys):
        """Returns (old values, status) in request order."""
        if self.world == 1 and not self.force_route:
            self.last_recv = keys.numel()
            return self.shard.delete(keys)
        return self._run(lambda k, v: self.shard.delete_part(k), keys, None, n_out=2,
                         begin=self.shard.delete_begin, end=self.shard.delete_end)

    def mixed(self, ops, keys, values):
        """Mixed batch (op codes 0 find / 1 insert / 2 delete, reading Q10).  The op
        codes travel with the keys; each owner runs its part as a mixed batch.
        Keys are distinct within the batch, so splitting it into chunks and
        shards changes no result.  Returns (values, status) in request order."""
        if self.world == 1 and not self.force_route:
            self.last_recv = keys.numel()
            return self.shard.mixed(ops, keys, values)
        return self._run(lambda k, v, t: self.shard.mixed(t, k, v), keys, values, n_out=2, tags=ops)

    def stats(self):
        return self.shard.stats()


class PeerRouter:
    """Fused dispatch / combine over peer memory (dyc_route_push / dyc_route_reply;
    DESIGN.md §7).  Each rank owns, in plain cudaMalloc buffers shared through
    CUDA IPC: a receive buffer of world * max_ops ops (17 B each, SoA), its uint64
    receive counter, and its result arrays (u32 values, u8 status) for up to
    max_ops ops.  A batch is

        push (every rank: hash, reserve, store ops into the owners' buffers)
        -> barrier -> owner: ONE local batch on the buffer in place, reply (results at
        the op's index in the requester's result arrays), reset counter
        -> barrier -> results are in request order.

    No counts are exchanged, nothing is unpermuted, and no NCCL data movement is
    used; the barriers are host barriers of the process group after a stream
    sync (they order the peer stores, which complete with their kernels)."""

    def __init__(self, dt, max_ops: int, buffer_factory=None, sync=None):
        """buffer_factory(nbytes) -> a PeerBuffer-like object and sync() (the
        stream sync before each barrier) default to table.PeerBuffer and a CUDA
        stream sync; the CPU tests inject shared-memory stand-ins."""
        import torch
        if buffer_factory is None:
            from .table import PeerBuffer as buffer_factory
        self._sync = sync if sync is not None else (lambda: torch.cuda.current_stream().synchronize())
        self.dt, self.max_ops = dt, max_ops
        W, r = dt.world, dt.rank
        self.cap = W * max_ops
        self.recv = buffer_factory(17 * self.cap)      # DYC_ROUTE_RECV_BYTES: keys | values | meta | tags
        self.cnt = buffer_factory(8)
        self.rv = buffer_factory(4 * max_ops)
        self.rs = buffer_factory(max_ops)
        bufs = (self.recv, self.cnt, self.rv, self.rs)
        mine = [b.handle() for b in bufs]
        allh = [None] * W
        dt.dist.all_gather_object(allh, mine, group=dt.group)
        ptrs = [[b.ptr for b in bufs] if w == r else [b.open(h) for b, h in zip(bufs, allh[w])] for w in range(W)]
        self.recv_p, self.cnt_p, self.rv_p, self.rs_p = ([p[i] for p in ptrs] for i in range(4))
        self.count = self.cnt.tensor(1, torch.int64)
        self.out_v = self.rv.tensor(max_ops, torch.int32)
        self.out_s = self.rs.tensor(max_ops, torch.uint8)
        self._barrier()

    def _barrier(self):
        self._sync()
        self.dt.dist.barrier(group=self.dt.group)

    def run(self, op, keys, values, n_out, begin, end, tags):
        dt = self.dt
        n = keys.numel()
        if n > self.max_ops:
            raise ValueError(f"batch of {n} ops exceeds the router's max_ops {self.max_ops}")
        dt.shard.route_push(keys, values, dt.world, dt.rank, self.recv_p, self.cnt_p, self.cap, tags=tags)
        self._barrier()
        m = int(self.count.item())
        if m > self.cap:
            raise RuntimeError(f"receive buffer overflow: {m} records > {self.cap}")
        dt.last_recv = m
        k, v, t = dt.shard.recv_views(self.recv, self.cap, m)    # the owner's batch, in place
        v = v if values is not None else None
        t = t if tags is not None else None
        if begin is not None:
            begin(m)
        res = op(k, v) if tags is None else op(k, v, t)
        res = res if isinstance(res, tuple) else (res,)
        if end is not None:
            end()
        if n_out == 1:
            dt.shard.route_reply(self.recv.ptr, self.cap, m, dt.world, status=res[0], out_status_ptrs=self.rs_p)
        else:
            dt.shard.route_reply(self.recv.ptr, self.cap, m, dt.world, vals=res[0], status=res[1],
                                 out_val_ptrs=self.rv_p, out_status_ptrs=self.rs_p)
        self.count.zero_()
        self._barrier()
        out_s = self.out_s[:n].clone()
        return out_s if n_out == 1 else (self.out_v[:n].clone(), out_s)

    def close(self):
        self.count = self.out_v = self.out_s = None       # views into the buffers go first
        for b in (self.recv, self.cnt, self.rv, self.rs):
            b.close()


# ---------------------------------------------------------------- bench (N > 1)
def bench_multi_gpu(args, rank, world, local, metric, ClockSampler, measured_peaks, run_oracle_sample,
                    compute_roofline=None):
    """Weak scaling: every rank issues one C2-shaped batch of its own keys (2^log2n
    inserts, 2^log2n finds at 50% hit, 2^(log2n-1) deletes) through the router;
    each shard receives ~1/G of every rank's ops.  Time = max over ranks."""
    import statistics
    import time
    import numpy as np
    import torch
    import torch.distributed as dist
    from . import workload as W
    from .table import Table

    from .sharded import ShardedTable, new_unique_id
    n = 1 << args.log2n
    cap, k_ins, v_ins, k_find, k_del = W.c2_rand_static_torch(args.log2n, device="cuda", key_base=rank * n,
                                                              miss_base=rank * n)
    p2p = getattr(args, "p2p", False)
    if p2p:
        # fused dispatch/combine over peer memory, orchestrated here
        shard = Table(d=4, init_capacity=cap, alpha=0.3, beta=0.85, bucket_slots=args.bucket_slots)
        dt = DistTable(shard, force_route=True, p2p=True, max_ops=n)
    else:
        # the sharded C ABI (dyc_dist_*): routing and NCCL exchange inside libdyc.so;
        # at N = 1 a one-rank communicator keeps the NCCL exchange on the path
        dt = ShardedTable(d=4, init_capacity=cap, alpha=0.3, beta=0.85, bucket_slots=args.bucket_slots,
                          unique_id=new_unique_id() if world == 1 else None)
        shard = dt
    stream = torch.cuda.current_stream()

    def step(evs=None):
        if evs: evs[0].record(stream)
        shard.clear()
        st = dt.insert(k_ins, v_ins)
        n_ins_recv = dt.last_recv
        if evs: evs[1].record(stream)
        v, f = dt.find(k_find)
        n_find_recv = dt.last_recv
        if evs: evs[2].record(stream)
        dv, ds = dt.delete(k_del)
        if evs: evs[3].record(stream)
        return st, f, ds, (n_ins_recv, n_find_recv, dt.last_recv)

    st, f, ds, recv = step()
    torch.cuda.synchronize()
    ok = torch.tensor([int((st == 1).all().item()), int(f.sum().item()), int(ds.sum().item())],
                      dtype=torch.int64, device="cuda")
    dist.all_reduce(ok)
    hit_rate = float(f.float().mean().item())
    # shard statistics for the roofline model (insert phase alone)
    shard.clear()
    dt.insert(k_ins, v_ins)
    s_ins = shard.stats()
    s_ins = s_ins[0] if isinstance(s_ins, list) else s_ins
    phi = s_ins["n_second_table"] / max(1, s_ins["m"])
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    dist.barrier()
    recs = []
    shard.launch_count(reset=True)
    shard.profile(True)
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
    launches = shard.launch_count()
    prof = shard.profile_read()
    shard.profile(False)
    ms = torch.tensor([a.elapsed_time(b) / args.steps], dtype=torch.float64, device="cuda")
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    ms_per_step = float(ms.item())
    n_ops = (n + n + n // 2) * world
    phases = {p: statistics.mean(r[i].elapsed_time(r[i + 1]) for r in recs)
              for i, p in enumerate(["insert", "find", "delete"])}
    roofline = None
    if compute_roofline is not None:
        roofline = compute_roofline(args, prof, n_ins=recv[0], n_find=recv[1], n_del=recv[2], s_ins=s_ins,
                                    hit_rate=hit_rate, phi=phi, phi_del=phi, cap=cap, stream=stream)
    # end to end: the rank's batch from pinned host memory, results back to the host
    e2e = None
    if not getattr(args, "no_e2e", False):
        pin = lambda t: t.cpu().pin_memory()  # noqa: E731
        hk, hv, hq, hd = pin(k_ins), pin(v_ins), pin(k_find), pin(k_del)
        o_st = torch.empty(n, dtype=torch.uint8, pin_memory=True)
        o_v, o_f = torch.empty(n, dtype=torch.int32, pin_memory=True), torch.empty(n, dtype=torch.uint8, pin_memory=True)
        o_dv, o_ds = (torch.empty(n // 2, dtype=torch.int32, pin_memory=True),
                      torch.empty(n // 2, dtype=torch.uint8, pin_memory=True))

        def e2e_step():
            shard.clear()
            o_st.copy_(dt.insert(hk.cuda(non_blocking=True), hv.cuda(non_blocking=True)), non_blocking=True)
            v, f = dt.find(hq.cuda(non_blocking=True))
            o_v.copy_(v, non_blocking=True)
            o_f.copy_(f, non_blocking=True)
            dv, ds = dt.delete(hd.cuda(non_blocking=True))
            o_dv.copy_(dv, non_blocking=True)
            o_ds.copy_(ds, non_blocking=True)
            torch.cuda.synchronize()
        e2e_step()
        dist.barrier()
        ts = []
        for _ in range(max(1, min(args.steps, 3))):
            t0 = time.perf_counter()
            e2e_step()
            ts.append(time.perf_counter() - t0)
        t = torch.tensor([statistics.mean(ts)], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e = {"value": n_ops / float(t.item()) / 1e6, "unit": "Mops/s",
               "h2d_bytes_per_step": 4 * n + 4 * n + 4 * n + 4 * (n // 2),
               "d2h_bytes_per_step": n + 5 * n + 5 * (n // 2), "ms_per_step": 1e3 * float(t.item()),
               "path": "pinned host batch -> sharded table (route, NCCL exchange, local kernels) -> host"}
    if rank != 0:
        return None
    return {
        "metric": metric, "value": n_ops / (ms_per_step * 1e-3) / 1e6, "unit": "Mops/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": f"C2-shaped batch per rank (2^{args.log2n} inserts, 2^{args.log2n} finds 50% hit, "
                               f"2^{args.log2n - 1} deletes), hash-partitioned over {world} shards, "
                               "routed to the owning shards", "d": 4, "alpha": 0.3, "beta": 0.85,
                   "bucket_slots": args.bucket_slots, "parallelism": f"shard{world}",
                   "routing": "p2p (fused push/reply over peer memory)" if p2p else
                   "dyc_dist_* C ABI: grouped ncclSend/ncclRecv inside libdyc.so",
                   "l2": "inputs and tables larger than L2; no flush needed"},
        "phase_ms_rank0": phases,
        "check": {"all_inserted_ranks": int(ok[0].item()), "found_total": int(ok[1].item()),
                  "deleted_total": int(ok[2].item()), "expected_found": world * n // 2,
                  "expected_deleted": world * n // 2},
        "gpu_launches": launches,
        "clocks": clk.summary(),
        "roofline": roofline, "cpu_baseline": None, "e2e": e2e,
    }


# ---------------------------------------------------------------- config C5
def bench_c5(args, rank, world, local, metric, ClockSampler):
    """Config C5 (BASELINE.json configs[4]): 2^31 RAND keys hash-partitioned over
    G shards.  Fill: global batches of 16M inserts of key(0 .. 2^31-1); then 32
    mixed 50/30/20 global batches of 16M ops.  Rank r issues ops [r*16M/G,
    (r+1)*16M/G) of every global batch; each shard starts at 1M slots and
    resizes on its own.  Time = max over ranks, per phase."""
    import torch
    import torch.distributed as dist
    from . import workload as W
    from .table import Table

    log2k = getattr(args, "c5_log2keys", 31)
    # 128 fill batches at every scale (2^31 keys: 16M per batch, the config);
    # keeps the 32 mixed batches' deletes below the live-find range at any scale
    from .sharded import ShardedTable, new_unique_id
    batch = 1 << min(24, log2k - 7)
    p2p = getattr(args, "p2p", False)
    if p2p:
        shard = Table(d=4, init_capacity=1 << 20, alpha=0.3, beta=0.85, bucket_slots=args.bucket_slots)
        dt = DistTable(shard, force_route=True, p2p=True, max_ops=(batch + world - 1) // world)
    else:
        routed = getattr(args, "routed", False)
        dt = ShardedTable(d=4, init_capacity=1 << 20, alpha=0.3, beta=0.85, bucket_slots=args.bucket_slots,
                          unique_id=new_unique_id() if (world == 1 and routed) else None)
        shard = dt
    stream = torch.cuda.current_stream()
    gen = W.c5_batches_torch(rank, world, device="cuda", log2_keys=log2k, batch=batch, mixed_batches=32)
    fill, mixed = [], []
    for item in gen:                      # materialise this rank's slices up front (inputs resident in HBM)
        (fill if item[0] == "insert" else mixed).append(item)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    checks = torch.zeros(4, dtype=torch.int64, device="cuda")
    # key(i) is a bijection of u32, so exactly one index maps to the reserved
    # EMPTY key (reading Q25: rejected with status INVALID, never stored)
    reserved = sum(int((k == -1).sum()) for _, k, _ in fill)
    exp_mixed = torch.zeros(2, dtype=torch.int64, device="cuda")   # valid (non-reserved) inserts, deletes
    for _, ops, k, _ in mixed:
        exp_mixed[0] += ((ops == 1) & (k != -1)).sum()
        exp_mixed[1] += ((ops == 2) & (k != -1)).sum()
    shard.profile(True)
    with ClockSampler(local) as clk:
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        a.record(stream)
        for _, k, v in fill:
            st = dt.insert(k, v)
            checks[0] += (st == 1).sum()
        b.record(stream)
        for _, ops, k, v in mixed:
            vals, st = dt.mixed(ops, k, v)
            checks[1] += ((ops == 0) & (st == 1)).sum()
            checks[2] += ((ops == 1) & (st == 1)).sum()
            checks[3] += ((ops == 2) & (st == 1)).sum()
        c.record(stream)
        torch.cuda.synchronize()
    t = torch.tensor([a.elapsed_time(b), b.elapsed_time(c)], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(checks)
    prof = shard.profile_read()
    shard.profile(False)
    st = shard.stats()
    st = st[0] if isinstance(st, list) else st
    fill_ms, mixed_ms = float(t[0]), float(t[1])
    r_t = torch.tensor([reserved], dtype=torch.int64, device="cuda")
    if world > 1:
        dist.all_reduce(r_t)
        dist.all_reduce(exp_mixed)
    reserved_all = int(r_t.item())
    n_fill, n_mixed = len(fill) * batch, len(mixed) * batch
    if rank != 0:
        return None
    return {
        "metric": metric, "value": (n_fill + n_mixed) / ((fill_ms + mixed_ms) * 1e-3) / 1e6, "unit": "Mops/s",
        "n_gpus": world, "steps": 1, "warmup": 0, "ms_per_step": fill_ms + mixed_ms, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": f"C5 RAND 2^{log2k} keys hash-partitioned over {world} shard(s): {len(fill)} global "
                               f"insert batches of {batch}, then {len(mixed)} mixed 50/30/20 batches of {batch}",
                   "d": 4, "alpha": 0.3, "beta": 0.85, "bucket_slots": args.bucket_slots,
                   "parallelism": f"shard{world}", "init_capacity_per_shard": 1 << 20,
                   "routing": "p2p (fused push/reply over peer memory)" if p2p else
                   ("dyc_dist_* C ABI: grouped ncclSend/ncclRecv inside libdyc.so"
                    if (world > 1 or getattr(args, "routed", False)) else "dyc_dist_* C ABI, one shard (no exchange)")},
        "phases": {"fill_ms": fill_ms, "fill_mops": n_fill / fill_ms / 1e3,
                   "mixed_ms": mixed_ms, "mixed_mops": n_mixed / mixed_ms / 1e3},
        "check": {"inserted_fill": int(checks[0]), "expected_fill": n_fill - reserved_all,
                  "reserved_key_in_fill": reserved_all,
                  "found_in_mixed": int(checks[1]), "expected_found": len(mixed) * (batch // 4),
                  "inserted_in_mixed": int(checks[2]), "expected_inserted_in_mixed": int(exp_mixed[0]),
                  "deleted_in_mixed": int(checks[3]), "expected_deleted_in_mixed": int(exp_mixed[1])},
        "shard0": {"fill": st["fill"], "buckets": st["buckets"], "m": st["m"], "n_upsize": st["n_upsize"], "n_device_alloc": st["n_device_alloc"], "alloc_ms": st["alloc_ms"],
                   "n_downsize": st["n_downsize"], "bytes": st["bytes_allocated"]},
        "kernel_ms_rank0": {k: round(v[0], 2) for k, v in prof.items() if v[1]},
        "kernel_calls_rank0": {k: v[1] for k, v in prof.items() if v[1]},
        "clocks": clk.summary(), "gpu_launches": sum(v[1] for v in prof.values()), "roofline": None,
        "cpu_baseline": None, "e2e": None,
    }
