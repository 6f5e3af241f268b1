"""Small end-to-end workloads for compute-sanitizer (memcheck, racecheck,
synccheck; scripts/gpu_pass.sh sanitize): C1, C3 and C4 streams at small
scale, the paper-weighted placement mode, a live resize window, the sharded C
ABI with local virtual shards, the chunk-staged path (forced), and the failure
path (max_hops = 1).  Every
batch is checked against the oracle so a sanitizer-clean run is also a correct
one.  Exits non-zero on a mismatch."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.sharded import ShardedTable  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import Table  # noqa: E402


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).cuda()


def hu(t):
    return t.cpu().numpy().view(np.uint32)


def run(g, o, batches, tag):
    for i, b in enumerate(batches):
        op = getattr(b, "op", "mixed")
        if op == "insert":
            ok = (g.insert(dev(b.keys), dev(b.values)).cpu().numpy() == o.insert(b.keys, b.values)).all()
        elif op == "find":
            v, f = g.find(dev(b.keys))
            ov, of = o.find(b.keys)
            ok = (f.cpu().numpy() == of).all() and (hu(v) == ov).all()
        elif op == "delete":
            v, s = g.delete(dev(b.keys))
            ov, os_ = o.delete(b.keys)
            ok = (s.cpu().numpy() == os_).all() and (hu(v) == ov).all()
        else:
            v, s = g.mixed(torch.from_numpy(b.ops).cuda(), dev(b.keys), dev(b.values))
            ov, os_ = o.mixed(b.ops, b.keys, b.values)
            ok = (s.cpu().numpy() == os_).all() and (hu(v) == ov).all()
        if not ok:
            raise SystemExit(f"{tag}: batch {i} differs from the oracle")
    if not (g.sorted_kv() == o.sorted_kv()).all():
        raise SystemExit(f"{tag}: contents differ")
    print(tag, "ok", flush=True)


def main():
    wl = W.c1_rand_small(n_keys=16384, batch=4096)
    mk = lambda **kw: (Table(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta, **kw),  # noqa: E731
                       oracle.OracleTable(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta,
                                          bucket_slots=8, **{k: v for k, v in kw.items() if k == "max_hops"}))
    run(*mk(), wl.batches, "C1")
    run(*mk(staged="force"), wl.batches, "C1-staged")     # chunk-staged path (TMA bulk copies, smem atomics)
    c3 = W.c3_dynamic(scale=0.0005, shape="RE", batch=4000, cycles=1, init_capacity=1024)
    g = Table(d=4, init_capacity=1024, alpha=0.3, beta=0.85)
    run(g, oracle.OracleTable(d=4, init_capacity=1024, alpha=0.3, beta=0.85, bucket_slots=8), c3.batches, "C3-RE")
    _, c4 = W.c4_zipf_mixed(U=40000, distinct=4000, grow_batches=4, cycles=1, init_capacity=1024)
    g = Table(d=4, init_capacity=1024, alpha=0.3, beta=0.85)
    run(g, oracle.OracleTable(d=4, init_capacity=1024, alpha=0.3, beta=0.85, bucket_slots=8), c4, "C4")
    g = Table(d=4, init_capacity=1024, alpha=0.3, beta=0.85, placement="paper_weighted")
    run(g, oracle.OracleTable(d=4, init_capacity=1024, alpha=0.3, beta=0.85, bucket_slots=8,
                              policy=oracle.PAPER_WEIGHTED), c3.batches[:30], "C3-RE weighted")
    rs = W.random_op_stream(77, n_batches=10, batch=3000, universe=6000, init_capacity=16)
    run(*mk(max_hops=1), rs.batches, "failure path")
    st = ShardedTable(d=4, init_capacity=1024, local_shards=3, rank=0, world=1)
    run(st, oracle.OracleTable(d=4, init_capacity=1024, alpha=0.3, beta=0.85, bucket_slots=8), c4, "sharded x3")
    # fused peer-memory routing (dyc_route_push / dyc_route_reply) with 3 virtual
    # shards on one GPU: insert, find and delete batches against the oracle
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
    from test_gpu_p2p import SEED, union_kv, virtual_batch
    shards = [Table(d=4, init_capacity=1024, alpha=0.3, beta=0.85, seed=SEED) for _ in range(3)]
    o = oracle.OracleTable(d=4, init_capacity=1024, alpha=0.3, beta=0.85, bucket_slots=8, seed=SEED)
    kk = W.key_range(0, 6000, 17)
    vv = W.val_of(kk, 0)
    st = virtual_batch(shards, lambda t, k, v, _: t.insert(k, v), dev(kk), dev(vv), n_out=1)
    if not (st.cpu().numpy() == o.insert(kk, vv)).all():
        raise SystemExit("p2p insert differs from the oracle")
    q = np.concatenate([kk[::2], W.key_range(1 << 31, 500, 17)])
    v, f = virtual_batch(shards, lambda t, k, v_, _: t.find(k), dev(q))
    ov, of = o.find(q)
    if not ((f.cpu().numpy() == of).all() and (hu(v) == ov).all()):
        raise SystemExit("p2p find differs from the oracle")
    v, st = virtual_batch(shards, lambda t, k, v_, _: t.delete(k), dev(kk[1::3]))
    if not (st.cpu().numpy() == o.delete(kk[1::3])[1]).all() or not (union_kv(shards) == o.sorted_kv()).all():
        raise SystemExit("p2p delete differs from the oracle")
    print("p2p x3 ok", flush=True)
    # live resize window (NEXT-1): finds and writes against a resize in flight
    g = Table(d=4, init_capacity=1 << 14, alpha=0.05, beta=0.9)
    o = oracle.OracleTable(d=4, init_capacity=1 << 14, alpha=0.05, beta=0.9, bucket_slots=8)
    k = W.key_range(0, 9000, 3)
    g.insert(dev(k), dev(W.val_of(k, 0)))
    o.insert(k, W.val_of(k, 0))
    side = torch.cuda.Stream()
    g.resize_begin(+1, resize_stream=side)
    o.resize(+1)
    k2 = W.key_range(1 << 20, 2000, 3)
    run(g, o, [W.Batch("find", k), W.Batch("insert", k2, W.val_of(k2, 1)), W.Batch("delete", k[:3000])], "live")
    g.resize_commit()
    torch.cuda.synchronize()
    print("all ok")


if __name__ == "__main__":
    main()
