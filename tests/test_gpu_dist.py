"""Sharding kernels (S11) on one GPU: G virtual shards through the CUDA routing
kernels, checked against the oracle's shard hash; and DistTable over a real
NCCL process group of size 1."""
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import Table  # noqa: E402


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).cuda()


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_route_kernels_partition_and_unpermute(oracle_mod, world):
    n = 300_001
    keys = W.key_range(0, n, 55)
    vals = W.val_of(keys, 2)
    g = Table(d=4, init_capacity=1024, seed=0x5EED0001)
    o = oracle_mod.OracleTable(d=4, init_capacity=1024, seed=0x5EED0001)
    shard = np.array([o.hash_x(5, int(k)) % world for k in keys[:20000]])   # x_{d+1} mod G
    kd, vd = dev(keys), dev(vals)
    counts = g.route_count(kd, world)
    kout, vout, pos = g.route_scatter(kd, vd, world, counts)
    c = counts.cpu().numpy()
    assert c.sum() == n
    ko = kout.cpu().numpy().view(np.uint32)
    vo = vout.cpu().numpy().view(np.uint32)
    p = pos.cpu().numpy().astype(np.int64)
    # every op lands once, with its value, in its shard's segment
    np.testing.assert_array_equal(ko[p], keys)
    np.testing.assert_array_equal(vo[p], vals)
    bounds = np.concatenate([[0], np.cumsum(c)])
    seg = np.searchsorted(bounds, p, side="right") - 1
    np.testing.assert_array_equal(seg[:20000], shard)
    np.testing.assert_array_equal(np.bincount(seg, minlength=world), c)
    # unpermute restores request order
    rv, rs = g.route_unpermute(pos, vout, (kout & 1).to(torch.uint8))
    np.testing.assert_array_equal(rv.cpu().numpy().view(np.uint32), vals)
    np.testing.assert_array_equal(rs.cpu().numpy(), (keys & 1).astype(np.uint8))


def test_dist_table_nccl_world1(oracle_mod):
    import torch.distributed as dist
    from paper_conf_icde_lizlhs21_b200.dist import DistTable
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1)
    try:
        wl = W.c2_rand_static(log2_n=16)
        ins, fnd, dele = wl.batches
        shard = Table(d=4, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta, bucket_slots=8)
        o = oracle_mod.OracleTable(d=4, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta,
                                   bucket_slots=8)
        dt = DistTable(shard, force_route=True)
        np.testing.assert_array_equal(dt.insert(dev(ins.keys), dev(ins.values)).cpu().numpy(),
                                      o.insert(ins.keys, ins.values))
        v, f = dt.find(dev(fnd.keys))
        ov, of = o.find(fnd.keys)
        np.testing.assert_array_equal(f.cpu().numpy(), of)
        np.testing.assert_array_equal(v.cpu().numpy().view(np.uint32), ov)
        v, st = dt.delete(dev(dele.keys))
        ov, os_ = o.delete(dele.keys)
        np.testing.assert_array_equal(st.cpu().numpy(), os_)
        np.testing.assert_array_equal(v.cpu().numpy().view(np.uint32), ov)
        np.testing.assert_array_equal(shard.sorted_kv(), o.sorted_kv())
    finally:
        dist.destroy_process_group()


def test_dist_table_mixed_routed_world1(oracle_mod):
    """DistTable.mixed through the CUDA routing kernels (op codes travel with the
    keys) equals the oracle's mixed batch (reading Q10)."""
    import torch.distributed as dist
    from paper_conf_icde_lizlhs21_b200.dist import DistTable
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1)
    try:
        meta, batches = W.c4_zipf_mixed(U=50000, distinct=5000, grow_batches=4, cycles=1, init_capacity=1024)
        shard = Table(d=4, init_capacity=1024, alpha=meta.alpha, beta=meta.beta, bucket_slots=8)
        o = oracle_mod.OracleTable(d=4, init_capacity=1024, alpha=meta.alpha, beta=meta.beta, bucket_slots=8)
        dt = DistTable(shard, force_route=True, chunks=3)
        for b in batches:
            v, st = dt.mixed(torch.from_numpy(b.ops).cuda(), dev(b.keys), dev(b.values))
            ov, os_ = o.mixed(b.ops, b.keys, b.values)
            np.testing.assert_array_equal(st.cpu().numpy(), os_)
            np.testing.assert_array_equal(v.cpu().numpy().view(np.uint32), ov)
            np.testing.assert_array_equal(shard.sorted_kv(), o.sorted_kv())
    finally:
        dist.destroy_process_group()


def test_bench_c5_small_checks(oracle_mod):
    """bench_c5 (config C5) at 2^20 keys on one shard: every fill key except the
    reserved one is INSERTED (reading Q25: key(i) is a bijection of u32, so one
    index maps to EMPTY), every live find hits, and the mixed inserts/deletes
    succeed exactly for the non-reserved keys."""
    import types
    import torch.distributed as dist
    from paper_conf_icde_lizlhs21_b200.dist import bench_c5
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()

    class NoClock:
        def __init__(self, *a):
            pass

        def __enter__(self):
            return self

        def __exit__(self, *a):
            return False

        def summary(self):
            return {}

    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1)
    try:
        args = types.SimpleNamespace(c5_log2keys=20, bucket_slots=8, routed=True, steps=1, warmup=0)
        out = bench_c5(args, 0, 1, 0, "m", NoClock)
    finally:
        dist.destroy_process_group()
    c = out["check"]
    assert c["inserted_fill"] == c["expected_fill"] == (1 << 20) - c["reserved_key_in_fill"]
    assert c["found_in_mixed"] == c["expected_found"]
    assert c["inserted_in_mixed"] == c["expected_inserted_in_mixed"]
    assert c["deleted_in_mixed"] == c["expected_deleted_in_mixed"]
