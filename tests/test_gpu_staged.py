"""Chunk-staged batches (dyc_staged.cuh, DESIGN.md §5 "Staged batches") against
the CPU oracle.

The staged path reorders a batch by the table chunk of each op's first-choice
bucket, applies it chunk by chunk in shared memory and
sends the ops their first-choice bucket cannot decide through the direct
kernels.  Results must be bit-exact with the oracle (the map semantics of
P:L188-189, batch model P:L464 with distinct keys, Q9): per-op statuses and
values, the sorted contents and the resize schedule after every batch; the
layout must satisfy I1/I2 under the oracle's hash.  DYC_STAGED_FORCE runs every
eligible batch staged whatever its size, so small oracle-friendly streams cover
the path, including updates, misses, the reserved key, deletes that clear the
first-choice-full invariant, and partially filled last chunks.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import Table  # noqa: E402

EMPTY = 0xFFFFFFFF


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).cuda()


def host_u32(t):
    return t.cpu().numpy().view(np.uint32)


def check_layout(g, o):
    kv, tb, bk = g.dump()
    st = g.stats()
    keys = (kv & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    assert o.check_layout(st["buckets"], keys, tb, bk) == 0, "I1/I2 violated on the GPU layout"
    assert sum(st["count"]) == st["m"] == kv.size, "I4: device counts != m"


def run_staged(oracle_mod, wl, staged="force", B=8, layout_every=True):
    g = Table(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta, bucket_slots=B,
              staged=staged)
    o = oracle_mod.OracleTable(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta,
                               bucket_slots=B)
    for i, b in enumerate(wl.batches):
        kd = dev(b.keys)
        if b.op == "insert":
            st = g.insert(kd, dev(b.values))
            np.testing.assert_array_equal(st.cpu().numpy(), o.insert(b.keys, b.values), err_msg=f"batch {i}")
        elif b.op == "find":
            v, f = g.find(kd)
            ov, of = o.find(b.keys)
            np.testing.assert_array_equal(f.cpu().numpy(), of, err_msg=f"batch {i} found")
            np.testing.assert_array_equal(host_u32(v), ov, err_msg=f"batch {i} values")
        else:
            v, st = g.delete(kd)
            ov, os_ = o.delete(b.keys)
            np.testing.assert_array_equal(st.cpu().numpy(), os_, err_msg=f"batch {i} delete status")
            np.testing.assert_array_equal(host_u32(v), ov, err_msg=f"batch {i} old values")
        np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv(), err_msg=f"contents after batch {i}")
        gs, os2 = g.stats(), o.stats()
        assert gs["m"] == os2["m"]
        if gs["n_fail_upsize"] == 0 and os2["n_fail_upsize"] == 0:
            assert gs["buckets"] == os2["buckets"], f"resize schedule diverged at batch {i}"
        if layout_every:
            check_layout(g, o)
    return g, o


@pytest.mark.parametrize("d", [2, 4, 8])
def test_staged_random_streams(oracle_mod, d):
    """Mixed insert (new keys and updates) / find (hits and misses) / delete
    batches, with up- and downsizes in between, every eligible batch staged."""
    alpha = round(min(0.3, 0.85 * d / (d + 1) - 0.01), 3)
    wl = W.random_op_stream(7100 + d, n_batches=40, batch=6000, universe=12000, d=d, alpha=alpha, beta=0.85,
                            init_capacity=64)
    g, _ = run_staged(oracle_mod, wl)
    s = g.stats()
    assert s["n_staged"] > 10, s["n_staged"]
    assert s["n_upsize"] > 0 and s["n_downsize"] > 0


def test_staged_edge_cases(oracle_mod):
    """Reserved key, updates, deletes of absent keys, one-op batches, and a table
    whose subtables end in partially filled chunks."""
    wl = W.Workload("edge", 4, 0.3, 0.85, 3000)
    ks = np.array([EMPTY, 1, 2, 3], dtype=np.uint32)
    wl.batches += [W.Batch("insert", ks, np.array([9, 10, 11, 12], dtype=np.uint32)),
                   W.Batch("find", np.array([EMPTY, 1, 5], dtype=np.uint32)),
                   W.Batch("insert", ks[1:], np.array([20, 21, 22], dtype=np.uint32)),
                   W.Batch("delete", np.array([EMPTY, 7, 2], dtype=np.uint32)),
                   W.Batch("find", np.array([2], dtype=np.uint32)),
                   W.Batch("insert", np.array([2], dtype=np.uint32), np.array([5], dtype=np.uint32))]
    big = W.key_range(0, 2500, 5)
    wl.batches += [W.Batch("insert", big, W.val_of(big, 1)), W.Batch("find", np.concatenate([big, big + 1])),
                   W.Batch("insert", big[::3], W.val_of(big[::3], 2)), W.Batch("delete", big[1::2]),
                   W.Batch("find", big), W.Batch("insert", big, W.val_of(big, 3))]
    g, _ = run_staged(oracle_mod, wl)
    assert g.stats()["n_staged"] >= 8


@pytest.mark.parametrize("log2_n", [18, 20])
def test_staged_c2_shape(oracle_mod, log2_n):
    """C2's shape (fill to 0.85, finds at 50% hit, deletes of half the keys) with
    the automatic choice: every batch is at least as large as the bucket count,
    so all three phases run staged, with many ops per bucket."""
    wl = W.c2_rand_static(log2_n=log2_n)
    g, o = run_staged(oracle_mod, wl, staged="auto" if log2_n >= 20 else "force", layout_every=False)
    check_layout(g, o)
    # automatic choice: the insert batch stages; finds stay direct; the delete
    # batch (n/2 ops) is below the automatic threshold at 2^20
    assert g.stats()["n_staged"] >= 1


def test_staged_matches_direct(oracle_mod):
    """The same stream with the staged path forced and switched off gives the
    same results and contents (both equal to the oracle's)."""
    wl = W.random_op_stream(9191, n_batches=25, batch=20000, universe=30000, init_capacity=4096)
    g1, _ = run_staged(oracle_mod, wl, staged="force", layout_every=False)
    g0, _ = run_staged(oracle_mod, wl, staged="off", layout_every=False)
    assert g0.stats()["n_staged"] == 0 and g1.stats()["n_staged"] > 0
    np.testing.assert_array_equal(g0.sorted_kv(), g1.sorted_kv())


def test_staged_not_used_for_other_bucket_widths(oracle_mod):
    wl = W.random_op_stream(55, n_batches=6, batch=3000, universe=6000, init_capacity=64)
    g, _ = run_staged(oracle_mod, wl, B=4)
    assert g.stats()["n_staged"] == 0


def test_staged_with_in_place_subtables(oracle_mod):
    """Subtables in reserved virtual ranges (DYC_RESIZE_IN_PLACE): the TMA bulk
    copies address the mapped range like any other device buffer."""
    wl = W.random_op_stream(4321, n_batches=16, batch=5000, universe=9000, init_capacity=512)
    g = Table(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta, bucket_slots=8,
              staged="force", in_place=True)
    o = oracle_mod.OracleTable(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta,
                               bucket_slots=8)
    for i, b in enumerate(wl.batches):
        kd = dev(b.keys)
        if b.op == "insert":
            np.testing.assert_array_equal(g.insert(kd, dev(b.values)).cpu().numpy(), o.insert(b.keys, b.values))
        elif b.op == "find":
            v, f = g.find(kd)
            ov, of = o.find(b.keys)
            np.testing.assert_array_equal(f.cpu().numpy(), of)
            np.testing.assert_array_equal(host_u32(v), ov)
        else:
            v, st = g.delete(kd)
            ov, os_ = o.delete(b.keys)
            np.testing.assert_array_equal(st.cpu().numpy(), os_)
            np.testing.assert_array_equal(host_u32(v), ov)
        np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv(), err_msg=f"contents after batch {i}")
    check_layout(g, o)
    assert g.stats()["n_staged"] > 0


def test_staged_not_used_with_paper_weighted_placement(oracle_mod):
    """The paper's balancing rule gives up the first-choice-full
    invariant the chunk pass decides misses with: its batches stay direct."""
    wl = W.random_op_stream(77, n_batches=8, batch=4000, universe=8000, init_capacity=64)
    g = Table(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta, bucket_slots=8,
              staged="force", placement="paper_weighted")
    o = oracle_mod.OracleTable(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta,
                               bucket_slots=8)
    for b in wl.batches:
        if b.op == "insert":
            np.testing.assert_array_equal(g.insert(dev(b.keys), dev(b.values)).cpu().numpy(),
                                          o.insert(b.keys, b.values))
        elif b.op == "find":
            v, f = g.find(dev(b.keys))
            np.testing.assert_array_equal(f.cpu().numpy(), o.find(b.keys)[1])
        else:
            v, st = g.delete(dev(b.keys))
            np.testing.assert_array_equal(st.cpu().numpy(), o.delete(b.keys)[1])
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
    assert g.stats()["n_staged"] == 0
