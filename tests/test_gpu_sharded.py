"""Parity of the sharded C ABI (dyc_dist_*) with the CPU
oracle: the routing, the exchange, the owners' batches and the unpermute all run
inside libdyc.so; this process only marshals arguments (sharded.py).

On one B200 the shards are local virtual shards (dyc_dist_create_ex with
local_shards = G), and the NCCL exchange is exercised with a one-rank
communicator (an id with world == 1: grouped ncclSend/ncclRecv to self).
Equality is the map semantics of P:L188-189: per-op statuses and values of
every batch, and the union of the shards' contents, equal the single-table
oracle's; each shard holds only keys with shard(k) = x_{d+1}(k) mod G equal to
its index, in a layout that is valid under the oracle's hash.
"""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.sharded import ShardedTable, new_unique_id  # noqa: E402

EMPTY = 0xFFFFFFFF


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).cuda()


def host_u32(t):
    return t.cpu().numpy().view(np.uint32)


def check_shards(st, o, G):
    a, b = o.hash_params()
    d = o.d
    for l in range(st.local_shards):
        sh = st.shard(l)
        kv, tb, bk = sh.dump()
        s = sh.stats()
        keys = (kv & np.uint64(0xFFFFFFFF)).astype(np.uint32)
        assert o.check_layout(s["buckets"], keys, tb, bk) == 0, f"shard {l}: I1/I2"
        assert sum(s["count"]) == s["m"] == kv.size
        x = ((np.uint64(a[d + 1]) * keys.astype(np.uint64)) % np.uint64(4294967291) + np.uint64(b[d + 1])) \
            % np.uint64(4294967291)
        owner = (x % np.uint64(G)).astype(np.int64)
        assert (owner == st.rank * st.local_shards + l).all(), f"shard {l} holds keys of another shard"


def run_stream(st, o, batches, check_every=1):
    for i, b in enumerate(batches):
        if b.op == "insert":
            got = st.insert(dev(b.keys), dev(b.values))
            np.testing.assert_array_equal(got.cpu().numpy(), o.insert(b.keys, b.values), err_msg=f"batch {i}")
        elif b.op == "find":
            v, f = st.find(dev(b.keys))
            ov, of = o.find(b.keys)
            np.testing.assert_array_equal(f.cpu().numpy(), of, err_msg=f"batch {i}")
            np.testing.assert_array_equal(host_u32(v), ov, err_msg=f"batch {i}")
        elif b.op == "delete":
            v, s = st.delete(dev(b.keys))
            ov, os_ = o.delete(b.keys)
            np.testing.assert_array_equal(s.cpu().numpy(), os_, err_msg=f"batch {i}")
            np.testing.assert_array_equal(host_u32(v), ov, err_msg=f"batch {i}")
        else:
            v, s = st.mixed(torch.from_numpy(b.ops).cuda(), dev(b.keys), dev(b.values))
            ov, os_ = o.mixed(b.ops, b.keys, b.values)
            np.testing.assert_array_equal(s.cpu().numpy(), os_, err_msg=f"batch {i}")
            np.testing.assert_array_equal(host_u32(v), ov, err_msg=f"batch {i}")
        if check_every and i % check_every == 0:
            np.testing.assert_array_equal(st.sorted_kv(), o.sorted_kv(), err_msg=f"contents after {i}")


class _Mixed:
    def __init__(self, mb):
        self.op, self.ops, self.keys, self.values = "mixed", mb.ops, mb.keys, mb.values


@pytest.mark.parametrize("G", [1, 3, 8])
def test_local_shards_random_stream(oracle_mod, G):
    wl = W.random_op_stream(5150 + G, n_batches=24, batch=4000, universe=9000, init_capacity=64)
    st = ShardedTable(d=4, init_capacity=64, alpha=wl.alpha, beta=wl.beta, local_shards=G, rank=0, world=1)
    o = oracle_mod.OracleTable(d=4, init_capacity=64, alpha=wl.alpha, beta=wl.beta, bucket_slots=8)
    run_stream(st, o, wl.batches)
    _, mixed = W.c4_zipf_mixed(U=30000, distinct=3000, grow_batches=4, cycles=1, init_capacity=64)
    run_stream(st, o, [_Mixed(m) for m in mixed])
    check_shards(st, o, G)
    per = [s["m"] for s in st.stats()]
    assert sum(per) == o.stats()["m"]
    if G > 1:
        assert min(per) > 0, "a virtual shard received nothing"
        assert any(s["n_upsize"] > 0 for s in st.stats()), "per-shard resizing never ran"


@pytest.mark.parametrize("G", [1, 4])
def test_nccl_self_exchange(oracle_mod, G):
    """The grouped ncclSend/ncclRecv path with a one-rank communicator: the
    same results as the oracle, C2-shaped batches with a ragged tail and an
    empty batch (a rank with nothing to send still joins the exchange)."""
    os.environ.setdefault("NCCL_SOCKET_IFNAME", "lo")
    wl = W.c2_rand_static(log2_n=16)
    more = W.key_range(1 << 30, 4321, 8)
    b0 = wl.batches[0]
    b0.keys = np.concatenate([b0.keys, more])
    b0.values = np.concatenate([b0.values, W.val_of(more, 0)])
    e = np.zeros(0, dtype=np.uint32)
    batches = [W.Batch("insert", e, e)] + wl.batches + [W.Batch("find", e)]
    st = ShardedTable(d=4, init_capacity=4096, alpha=0.3, beta=0.85, local_shards=G, rank=0, world=1,
                      unique_id=new_unique_id())
    o = oracle_mod.OracleTable(d=4, init_capacity=4096, alpha=0.3, beta=0.85, bucket_slots=8)
    run_stream(st, o, batches)
    check_shards(st, o, G)


def test_sharded_argument_errors():
    from paper_conf_icde_lizlhs21_b200._lib import DycError
    st = ShardedTable(d=4, init_capacity=4096, local_shards=2, rank=0, world=1)
    with pytest.raises(DycError):
        st.shard(2)
    with pytest.raises(DycError):
        ShardedTable(d=4, init_capacity=4096, local_shards=0, rank=0, world=1)
    with pytest.raises(DycError):
        ShardedTable(d=4, init_capacity=4096, rank=2, world=2, unique_id=b"\0" * 128)
