"""Fused routing over peer memory (S11): dyc_route_push (hash,
reserve, store ops into the owners' receive buffers) and dyc_route_reply
(results stored at the op's index in the requester's arrays).

1. G virtual shards on one GPU: every "rank" pushes its slice of a batch into
   all G receive buffers (local pointers), every owner runs its received ops as
   one batch in place and replies; per-op results and the union of the shards' contents
   must equal the single-table oracle (ops on different keys never interact).
2. Two processes on cuda:0 (gloo process group): DistTable(p2p=True) with the
   receive/result buffers mapped through real CUDA IPC handles.
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import PeerBuffer, Table  # noqa: E402

SEED = 0x5EED0077


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).cuda()


def virtual_batch(shards, op, keys, vals=None, tags=None, n_out=2):
    """One batch through push -> owner batch -> reply with G shards on one GPU."""
    G = len(shards)
    n = keys.numel()
    cuts = [n * r // G for r in range(G + 1)]
    cap = n + 1
    recv = [PeerBuffer(17 * cap) for _ in range(G)]
    cnt = [PeerBuffer(8) for _ in range(G)]
    out_v = torch.full((n,), 7, dtype=torch.int32, device="cuda")
    out_s = torch.full((n,), 9, dtype=torch.uint8, device="cuda")
    try:
        for r in range(G):
            lo, hi = cuts[r], cuts[r + 1]
            shards[r].route_push(keys[lo:hi], vals[lo:hi] if vals is not None else None, G, r,
                                 [b.ptr for b in recv], [c.ptr for c in cnt], cap,
                                 tags=tags[lo:hi] if tags is not None else None)
        torch.cuda.synchronize()
        counts = [int(c.tensor(1, torch.int64).item()) for c in cnt]
        assert sum(counts) == n
        # requester r's result arrays start at its slice of the batch result
        vp = [out_v.data_ptr() + 4 * cuts[r] for r in range(G)]
        sp = [out_s.data_ptr() + cuts[r] for r in range(G)]
        for s in range(G):
            m = counts[s]
            k, v, t = Table.recv_views(recv[s], cap, m)
            v = v if vals is not None else None
            t = t if tags is not None else None
            # every record routed here hashes to this shard
            if m:
                dest = shards[s].route_count(k, G).cpu().numpy()
                assert dest[s] == m
            res = op(shards[s], k, v, t)
            res = res if isinstance(res, tuple) else (res,)
            if n_out == 1:
                Table.route_reply(recv[s].ptr, cap, m, G, status=res[0], out_status_ptrs=sp)
            else:
                Table.route_reply(recv[s].ptr, cap, m, G, vals=res[0], status=res[1], out_val_ptrs=vp,
                                  out_status_ptrs=sp)
        torch.cuda.synchronize()
    finally:
        for b in recv + cnt:
            b.close()
    return out_s if n_out == 1 else (out_v, out_s)


def by_key(kv):
    """Packed slots ordered by key (the low 32 bits), as sorted_kv() returns them."""
    return kv[np.argsort((kv & np.uint64(0xFFFFFFFF)).astype(np.uint32), kind="stable")]


def union_kv(shards):
    return by_key(np.concatenate([s.sorted_kv() for s in shards]))


@pytest.mark.parametrize("G", [1, 3, 8])
def test_p2p_virtual_shards_c2(oracle_mod, G):
    wl = W.c2_rand_static(log2_n=15)
    ins, fnd, dele = wl.batches
    shards = [Table(d=4, init_capacity=1024, alpha=wl.alpha, beta=wl.beta, bucket_slots=8, seed=SEED)
              for _ in range(G)]
    o = oracle_mod.OracleTable(d=4, init_capacity=1024, alpha=wl.alpha, beta=wl.beta, bucket_slots=8, seed=SEED)
    st = virtual_batch(shards, lambda sh, k, v, t: sh.insert(k, v), dev(ins.keys), dev(ins.values), n_out=1)
    np.testing.assert_array_equal(st.cpu().numpy(), o.insert(ins.keys, ins.values))
    v, f = virtual_batch(shards, lambda sh, k, v, t: sh.find(k), dev(fnd.keys))
    ov, of = o.find(fnd.keys)
    np.testing.assert_array_equal(f.cpu().numpy(), of)
    np.testing.assert_array_equal(v.cpu().numpy().view(np.uint32), ov)
    v, s = virtual_batch(shards, lambda sh, k, v, t: sh.delete(k), dev(dele.keys))
    ov, os_ = o.delete(dele.keys)
    np.testing.assert_array_equal(s.cpu().numpy(), os_)
    np.testing.assert_array_equal(v.cpu().numpy().view(np.uint32), ov)
    np.testing.assert_array_equal(union_kv(shards), o.sorted_kv())


def test_p2p_virtual_shards_mixed_zipf(oracle_mod):
    """C4-shaped mixed batches: the op code travels in the record's tag byte."""
    G = 4
    meta, batches = W.c4_zipf_mixed(U=40000, distinct=4000, grow_batches=3, cycles=1, init_capacity=1024)
    shards = [Table(d=4, init_capacity=1024, alpha=meta.alpha, beta=meta.beta, bucket_slots=8, seed=SEED)
              for _ in range(G)]
    o = oracle_mod.OracleTable(d=4, init_capacity=1024, alpha=meta.alpha, beta=meta.beta, bucket_slots=8, seed=SEED)
    for b in batches:
        v, st = virtual_batch(shards, lambda sh, k, v, t: sh.mixed(t, k, v), dev(b.keys), dev(b.values),
                              tags=torch.from_numpy(b.ops).cuda())
        ov, os_ = o.mixed(b.ops, b.keys, b.values)
        np.testing.assert_array_equal(st.cpu().numpy(), os_)
        np.testing.assert_array_equal(v.cpu().numpy().view(np.uint32), ov)
    np.testing.assert_array_equal(union_kv(shards), o.sorted_kv())


def test_p2p_push_overflow_is_detected():
    """Records past recv_cap are dropped and the counter still counts them."""
    sh = Table(d=4, init_capacity=1024, seed=SEED)
    keys = dev(W.key_range(0, 5000, 3))
    recv, cnt = PeerBuffer(17 * 100), PeerBuffer(8)
    try:
        sh.route_push(keys, None, 1, 0, [recv.ptr], [cnt.ptr], 100)
        torch.cuda.synchronize()
        assert int(cnt.tensor(1, torch.int64).item()) == 5000
        with pytest.raises(Exception):
            sh.route_push(keys, None, 1, 1, [recv.ptr], [cnt.ptr], 100)     # src_rank >= world
    finally:
        recv.close()
        cnt.close()


# ------------------------------------------------------------ two processes
def _worker(rank, world, port, log2n, result_dir):
    import torch.distributed as dist
    import oracle
    from paper_conf_icde_lizlhs21_b200.dist import DistTable
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        wl = W.c2_rand_static(log2_n=log2n)
        ins, fnd, dele = wl.batches
        n = len(ins.keys)
        cut = lambda a: a[n * rank // world:n * (rank + 1) // world] if len(a) == n else \
            a[len(a) * rank // world:len(a) * (rank + 1) // world]
        shard = Table(d=4, init_capacity=1024, alpha=wl.alpha, beta=wl.beta, bucket_slots=8, seed=SEED)
        dt = DistTable(shard, force_route=True, p2p=True, max_ops=n)
        st = dt.insert(dev(cut(ins.keys)), dev(cut(ins.values))).cpu().numpy()
        v, f = dt.find(dev(cut(fnd.keys)))
        dv, ds = dt.delete(dev(cut(dele.keys)))
        torch.cuda.synchronize()
        mine = {"st": st, "v": v.cpu().numpy(), "f": f.cpu().numpy(), "dv": dv.cpu().numpy(),
                "ds": ds.cpu().numpy(), "kv": shard.sorted_kv()}
        allp = [None] * world
        dist.all_gather_object(allp, mine)
        dt.p2p.close()
        if rank == 0:
            o = oracle.OracleTable(d=4, init_capacity=1024, alpha=wl.alpha, beta=wl.beta, bucket_slots=8, seed=SEED)
            np.testing.assert_array_equal(np.concatenate([p["st"] for p in allp]), o.insert(ins.keys, ins.values))
            ov, of = o.find(fnd.keys)
            np.testing.assert_array_equal(np.concatenate([p["f"] for p in allp]), of)
            np.testing.assert_array_equal(np.concatenate([p["v"] for p in allp]).view(np.uint32), ov)
            ov, os_ = o.delete(dele.keys)
            np.testing.assert_array_equal(np.concatenate([p["ds"] for p in allp]), os_)
            np.testing.assert_array_equal(np.concatenate([p["dv"] for p in allp]).view(np.uint32), ov)
            np.testing.assert_array_equal(by_key(np.concatenate([p["kv"] for p in allp])), o.sorted_kv())
            open(os.path.join(result_dir, "ok"), "w").write("ok")
    finally:
        dist.destroy_process_group()


def test_p2p_two_processes_ipc(tmp_path, oracle_mod):
    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    mp.spawn(_worker, args=(2, port, 14, str(tmp_path)), nprocs=2, join=True)
    assert (tmp_path / "ok").exists()


def test_p2p_entry_points_reject_bad_arguments():
    """Argument checks of the peer-routing C ABI (include/dycuckoo.h)."""
    import ctypes as C
    from paper_conf_icde_lizlhs21_b200 import _lib as L
    sh = Table(d=4, init_capacity=1024, seed=SEED)
    keys = dev(W.key_range(0, 100, 5))
    recv, cnt = PeerBuffer(17 * 128), PeerBuffer(8)
    lib = L.load_library()
    try:
        with pytest.raises(ValueError):                       # pointer list shorter than world
            sh.route_push(keys, None, 2, 0, [recv.ptr], [cnt.ptr], 128)
        arr = lambda ps: C.cast((C.c_void_p * len(ps))(*ps), C.c_void_p)  # noqa: E731
        s = torch.cuda.current_stream().cuda_stream
        for world in (0, 65):
            assert lib.dyc_route_push(sh.handle, keys.data_ptr(), None, None, 100, world, 0,
                                      arr([recv.ptr] * 65), arr([cnt.ptr] * 65), 128, s) == L.DYC_ERR_INVALID_ARG
        assert lib.dyc_route_push(sh.handle, keys.data_ptr(), None, None, 100, 1, 0, arr([0]), arr([cnt.ptr]),
                                  128, s) == L.DYC_ERR_INVALID_ARG          # null peer pointer
        st = torch.zeros(100, dtype=torch.uint8, device="cuda")
        # a result array without destinations, and n > recv_cap
        assert lib.dyc_route_reply(recv.ptr, 128, 100, None, st.data_ptr(), 1, None, None, s) == L.DYC_ERR_INVALID_ARG
        assert lib.dyc_route_reply(recv.ptr, 128, 129, None, st.data_ptr(), 1, None, arr([st.data_ptr()]),
                                   s) == L.DYC_ERR_INVALID_ARG
        assert lib.dyc_ipc_alloc(0, C.byref(C.c_void_p())) == L.DYC_ERR_INVALID_ARG
        assert lib.dyc_ipc_get_handle(None, None) == L.DYC_ERR_INVALID_ARG
        # n == 0 is a no-op
        assert lib.dyc_route_push(sh.handle, keys.data_ptr(), None, None, 0, 1, 0, arr([recv.ptr]), arr([cnt.ptr]),
                                  128, s) == L.DYC_OK
    finally:
        recv.close()
        cnt.close()
