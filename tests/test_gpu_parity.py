"""Parity of the CUDA path (libdyc.so through its C ABI) with the CPU oracle.

Bit-exact on: per-op statuses, find values, sorted contents after EVERY batch,
subtable sizes after every batch (the resize schedule; valid while neither side
needed a failure-triggered upsize), and the hash specification (test vectors).
Placement (which slot, which of the two tables) is nondeterministic on the GPU:
instead the GPU layout is checked for validity with the oracle's hash (I1, I2).
"""
import os

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


def make_pair(oracle_mod, wl, B=4, max_hops=64, seed=0x5EED0001):
    g = Table(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta,
              bucket_slots=B, max_hops=max_hops, seed=seed)
    o = oracle_mod.OracleTable(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta,
                               bucket_slots=B, max_hops=max_hops, seed=seed)
    return g, o


def check_layout(g, o):
    kv, tb, bk = g.dump()
    st = g.stats()
    keys = (kv & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    assert o.check_layout(st["buckets"], keys, tb, bk) == 0, "I1/I2 violated on the GPU layout"
    assert sum(st["count"]) == st["m"] == kv.size, "I4: device counts != m"


def run_parity(oracle_mod, wl, B=4, max_hops=64, layout_every=True, compare_sizes=True):
    g, o = make_pair(oracle_mod, wl, B=B, max_hops=max_hops)
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
        if compare_sizes and gs["n_fail_upsize"] == 0 and os2["n_fail_upsize"] == 0:
            assert gs["buckets"] == os2["buckets"], f"resize schedule diverged at batch {i}"
        assert max(gs["buckets"]) <= 2 * min(gs["buckets"]), "I6 (P:L312)"
        assert gs["m"] <= wl.beta * gs["N"], "I5 upper"
        if layout_every:
            check_layout(g, o)
    return g, o


# ------------------------------------------------------------------ hash spec
def test_hash_matches_golden_vectors():
    path = os.path.join(os.path.dirname(__file__), "golden", "hash_vectors.txt")
    rows = [l.split() for l in open(path) if l.strip() and not l.startswith("#")]
    seed = [int(l.split()[2], 0) for l in open(path) if l.startswith("# seed")][0]
    g = Table(d=4, init_capacity=4 * 4 * 1000, seed=seed)
    keys = np.array([int(r[0]) for r in rows], dtype=np.uint32)
    x, pr = g.hash_probe(dev(keys))
    x = x.cpu().numpy().view(np.uint32)
    pr = pr.cpu().numpy()
    for j, r in enumerate(rows):
        assert x[j].tolist() == [int(v) for v in r[1:7]], f"key {r[0]}"
        assert pr[j].tolist() == [int(r[7]), int(r[8])]


def test_hash_params_match_oracle(oracle_mod):
    g = Table(d=6, init_capacity=1000, seed=1234567)
    o = oracle_mod.OracleTable(d=6, init_capacity=1000, seed=1234567)
    ga, gb = g.hash_params()
    oa, ob = o.hash_params()
    np.testing.assert_array_equal(ga, oa)
    np.testing.assert_array_equal(gb, ob)


# ------------------------------------------------------------------ configs
@pytest.mark.parametrize("seed", [None, 0xD7C10001, 0xD7C10002])
def test_c1_parity_every_batch(oracle_mod, seed):
    """Config C1 (BASELINE.json configs[0]) end to end, three seeds (SURVEY
    §8(d): correctness runs use three); 17 upsizes, 49 downsizes (the schedule
    depends on m only, so on no seed)."""
    g, o = run_parity(oracle_mod, W.c1_rand_small(seed_cfg=seed))
    s = g.stats()
    assert (s["n_upsize"], s["n_downsize"], s["n_fail_upsize"]) == (17, 49, 0)
    assert s["buckets"] == [1, 1, 1, 1] and s["m"] == 0


@pytest.mark.parametrize("log2_n,extra,seed", [(16, 0, None), (16, 777, 0xD7C20001), (16, 31, 0xD7C20002),
                                               (20, 12345, None)])
def test_c2_shape_parity(oracle_mod, log2_n, extra, seed):
    """Config C2's shape at oracle-friendly sizes, with a ragged tail; three seeds at 2^16."""
    wl = W.c2_rand_static(log2_n=log2_n, seed_cfg=seed)
    if extra:
        more = W.key_range(1 << 30, extra, 99)
        b0 = wl.batches[0]
        b0.keys = np.concatenate([b0.keys, more])
        b0.values = np.concatenate([b0.values, W.val_of(more, 0)])
    g, o = run_parity(oracle_mod, wl, layout_every=(log2_n <= 16))
    check_layout(g, o)


@pytest.mark.parametrize("B", [4, 8, 16, 32])
@pytest.mark.parametrize("d", [2, 4, 7])
def test_random_streams_parity(oracle_mod, B, d):
    alpha = round(min(0.3, 0.85 * d / (d + 1) - 0.01), 3)
    wl = W.random_op_stream(1000 + 10 * d + B, n_batches=30, batch=3000, universe=6000, d=d,
                            alpha=alpha, beta=0.85, init_capacity=64)
    g, _ = run_parity(oracle_mod, wl, B=B)
    s = g.stats()
    assert s["n_upsize"] > 0 and s["n_downsize"] > 0


def test_failure_path_keeps_every_key(oracle_mod):
    """max_hops = 1 forces failed chains: retry + failure upsizes, never a
    lost or duplicated key."""
    wl = W.random_op_stream(4242, n_batches=20, batch=4000, universe=8000, init_capacity=16)
    g, _ = run_parity(oracle_mod, wl, B=4, max_hops=1, compare_sizes=False)


def test_edge_cases(oracle_mod):
    wl = W.Workload("edge", 4, 0.3, 0.85, 64)
    e = np.zeros(0, dtype=np.uint32)
    ks = np.array([EMPTY, 1, 2, 3], dtype=np.uint32)
    wl.batches += [W.Batch("insert", e, e), W.Batch("find", e), W.Batch("delete", e),
                   W.Batch("insert", ks, np.array([9, 10, 11, 12], dtype=np.uint32)),
                   W.Batch("find", np.array([EMPTY, 1, 5], dtype=np.uint32)),
                   W.Batch("insert", ks[1:], np.array([20, 21, 22], dtype=np.uint32)),   # updates
                   W.Batch("delete", np.array([EMPTY, 7, 2], dtype=np.uint32)),
                   W.Batch("find", np.array([2, 3, 0], dtype=np.uint32))]
    # a batch far bigger than the table: several upsizes inside one insert
    big = W.key_range(0, 50000, 5)
    wl.batches.append(W.Batch("insert", big, W.val_of(big, 1)))
    wl.batches.append(W.Batch("delete", big[:49990]))
    run_parity(oracle_mod, wl)


def test_example2_scenario_semantics(oracle_mod):
    """Example 2 as one GPU batch: k1 into a free bucket, k33 updated
    in place, k65 evicting from a full bucket; every key ends present once."""
    keys = W.key_range(0, 40, 77)
    # fill a tiny table so inserts must evict, then insert/update a mix
    g = Table(d=4, init_capacity=64, bucket_slots=4, alpha=0.01, beta=0.99)
    o = oracle_mod.OracleTable(d=4, init_capacity=64, bucket_slots=4, alpha=0.01, beta=0.99)
    first = keys[:30]
    g.insert(dev(first), dev(W.val_of(first, 0)))
    o.insert(first, W.val_of(first, 0))
    mix = np.concatenate([keys[30:40], first[:5]])
    st = g.insert(dev(mix), dev(W.val_of(mix, 3)))
    np.testing.assert_array_equal(st.cpu().numpy(), o.insert(mix, W.val_of(mix, 3)))
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
    check_layout(g, o)


# ------------------------------------------------------------------ resize kernels
def _filled_table(oracle_mod, n=60000, B=4):
    g = Table(d=4, init_capacity=int(n / 0.8), alpha=0.05, beta=0.95, bucket_slots=B)
    o = oracle_mod.OracleTable(d=4, init_capacity=int(n / 0.8), alpha=0.05, beta=0.95, bucket_slots=B)
    k = W.key_range(0, n, 31)
    g.insert(dev(k), dev(W.val_of(k, 0)))
    o.insert(k, W.val_of(k, 0))
    return g, o


@pytest.mark.parametrize("B", [4, 16])
def test_upsize_split_property_gpu(oracle_mod, B):
    """P:L377-381 on the GPU kernel: entries of bucket b land in b or b+n."""
    g, o = _filled_table(oracle_mod, B=B)
    kv0, tb0, bk0 = g.dump()
    n0 = g.stats()["buckets"]
    g.resize(+1)
    kv1, tb1, bk1 = g.dump()
    assert g.stats()["buckets"][0] == 2 * n0[0]
    before = {int(x & 0xFFFFFFFF): (int(a), int(b)) for x, a, b in zip(kv0, tb0, bk0)}
    after = {int(x & 0xFFFFFFFF): (int(a), int(b)) for x, a, b in zip(kv1, tb1, bk1)}
    assert before.keys() == after.keys()
    for k, (t, b) in before.items():
        if t == 0:
            assert after[k] in ((0, b), (0, b + n0[0]))
        else:
            assert after[k] == (t, b)
    np.testing.assert_array_equal(np.sort(kv0), np.sort(kv1))
    check_layout(g, o)


@pytest.mark.parametrize("B", [4, 8])
def test_downsize_residuals_gpu(oracle_mod, B):
    """P:L387-395 on the GPU kernels: contents unchanged, residual count equals
    sum_b' max(0, |b'|+|b'+h|-B) from the pre-resize dump."""
    g, o = _filled_table(oracle_mod, n=30000, B=B)
    g.resize(+1)
    g.resize(+1)
    kv0, tb0, bk0 = g.dump()
    s0 = g.stats()
    t = 1
    h = s0["buckets"][t] // 2
    occ = np.bincount(bk0[tb0 == t].astype(np.int64), minlength=2 * h)
    expect = int(np.maximum(0, occ[:h] + occ[h:] - B).sum())
    g.resize(-1)
    s1 = g.stats()
    assert s1["buckets"][t] == h
    assert s1["n_residual"] - s0["n_residual"] == expect
    np.testing.assert_array_equal(np.sort(kv0), np.sort(g.dump()[0]))
    check_layout(g, o)


@pytest.mark.parametrize("method", [1, 2])
@pytest.mark.parametrize("direction", [+1, -1])
def test_resize_baselines_keep_contents(oracle_mod, method, direction):
    g, o = _filled_table(oracle_mod, n=40000)
    if direction < 0:
        g.resize(+1)
    kv0 = np.sort(g.dump()[0])
    g.resize(direction, -1, method)
    np.testing.assert_array_equal(kv0, np.sort(g.dump()[0]))
    check_layout(g, o)


def test_resize_refusals():
    from paper_conf_icde_lizlhs21_b200._lib import DycError
    g = Table(d=4, init_capacity=4 * 4 * 8)
    g.resize(+1, 0)
    with pytest.raises(DycError):
        g.resize(+1, 0)
    with pytest.raises(DycError):
        g.resize(-1, 3)


# ------------------------------------------------------------------ host-buffer path
def test_host_entry_points_match_device(oracle_mod):
    wl = W.c2_rand_static(log2_n=15)
    g = Table(d=4, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta, bucket_slots=8)
    o = oracle_mod.OracleTable(d=4, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta,
                               bucket_slots=8)
    ins, fnd, dele = wl.batches
    np.testing.assert_array_equal(g.insert_host(ins.keys, ins.values), o.insert(ins.keys, ins.values))
    v, f = g.find_host(fnd.keys)
    ov, of = o.find(fnd.keys)
    np.testing.assert_array_equal(f, of)
    np.testing.assert_array_equal(v, ov)
    v, s = g.delete_host(dele.keys)
    ov, os_ = o.delete(dele.keys)
    np.testing.assert_array_equal(s, os_)
    np.testing.assert_array_equal(v, ov)
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())


def test_host_entry_points_chunked(oracle_mod):
    """The host-buffer path pipelines 2^22-op chunks: a batch spanning several
    chunks with a ragged tail gives the oracle's results."""
    n = (1 << 22) * 2 + 12345
    keys = W.key_range(0, n, 321)
    vals = W.val_of(keys, 0)
    g = Table(d=4, init_capacity=int(n / 0.8), alpha=0.3, beta=0.85, bucket_slots=8)
    o = oracle_mod.OracleTable(d=4, init_capacity=int(n / 0.8), alpha=0.3, beta=0.85, bucket_slots=8)
    np.testing.assert_array_equal(g.insert_host(keys, vals), o.insert(keys, vals))
    upd = keys[::3].copy()
    np.testing.assert_array_equal(g.insert_host(upd, W.val_of(upd, 1)), o.insert(upd, W.val_of(upd, 1)))
    q = np.concatenate([keys[::2], W.key_range(1 << 31, n // 2, 321)])
    v, f = g.find_host(q)
    ov, of = o.find(q)
    np.testing.assert_array_equal(f, of)
    np.testing.assert_array_equal(v, ov)
    dk = keys[1::2].copy()
    v, s = g.delete_host(dk)
    ov, os_ = o.delete(dk)
    np.testing.assert_array_equal(s, os_)
    np.testing.assert_array_equal(v, ov)
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
    assert g.stats()["buckets"] == o.stats()["buckets"]


# ------------------------------------------------------------------ full size (C2)
@pytest.mark.slow
def test_c2_full_size_sampled():
    """BASELINE.json configs[1] at full size (2^27 keys, fill 0.85), in the
    launch configuration bench.py times.  Expected results follow from the
    generator: hits return val(k,0), misses NOT_FOUND; every delete hits; the
    table never resizes; the final dump holds exactly the undeleted keys
    (checked on a sample of 2^20 keys one by one)."""
    wl = W.c2_rand_static(log2_n=27)
    ins, fnd, dele = wl.batches
    g = Table(d=4, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta, bucket_slots=8)
    st = g.insert(dev(ins.keys), dev(ins.values))
    assert int((st == 1).sum()) == ins.keys.size
    s = g.stats()
    assert s["m"] == ins.keys.size and s["n_upsize"] == 0 and sum(s["count"]) == s["m"]
    assert abs(s["fill"] - 0.85) < 1e-3
    v, f = g.find(dev(fnd.keys))
    f = f.cpu().numpy()
    v = host_u32(v)
    live = np.isin(fnd.keys, ins.keys)
    np.testing.assert_array_equal(f.astype(bool), live)
    np.testing.assert_array_equal(v[live], W.val_of(fnd.keys[live], 0))
    assert (v[~live] == EMPTY).all()
    vd, sd = g.delete(dev(dele.keys))
    assert (sd.cpu().numpy() == 1).all()
    np.testing.assert_array_equal(host_u32(vd), W.val_of(dele.keys, 0))
    s = g.stats()
    assert s["m"] == ins.keys.size - dele.keys.size and s["n_downsize"] == 0
    rng = np.random.Generator(np.random.PCG64(5))
    sample = ins.keys[rng.choice(ins.keys.size, size=1 << 20, replace=False)]
    v, f = g.find(dev(sample))
    deleted = np.isin(sample, dele.keys)
    np.testing.assert_array_equal(f.cpu().numpy().astype(bool), ~deleted)
    np.testing.assert_array_equal(host_u32(v)[~deleted], W.val_of(sample[~deleted], 0))


# ------------------------------------------------------------------ dynamic configs
@pytest.mark.parametrize("shape,seed", [("TW", None), ("RE", None), ("TW", 0xD7C30001), ("RE", 0xD7C30002)])
def test_c3_dynamic_parity(oracle_mod, shape, seed):
    """Config C3's shape (sliding window, swap pass, two cycles) at small scale:
    up- and downsizes repeat; contents and the resize schedule match every batch."""
    wl = W.c3_dynamic(scale=0.001, shape=shape, batch=5000, cycles=2, init_capacity=1024, seed_cfg=seed)
    g, o = run_parity(oracle_mod, wl, B=8, layout_every=False)
    check_layout(g, o)
    s = g.stats()
    assert s["n_upsize"] > 0 and s["n_downsize"] > 0


@pytest.mark.parametrize("seed", [None, 0xD7C40001, 0xD7C40002])
def test_c4_zipf_mixed_parity(oracle_mod, seed):
    """Config C4's shape: Zipf(0.99) mixed 50/30/20 batches through dyc_mixed_batch
    (reading Q10: find -> insert -> delete), grow then drain, two cycles; three seeds."""
    meta, batches = W.c4_zipf_mixed(U=60000, distinct=6000, grow_batches=6, cycles=2, init_capacity=1024,
                                    seed_cfg=seed)
    g = Table(d=4, init_capacity=meta.init_capacity, alpha=meta.alpha, beta=meta.beta, bucket_slots=8)
    o = oracle_mod.OracleTable(d=4, init_capacity=meta.init_capacity, alpha=meta.alpha, beta=meta.beta,
                               bucket_slots=8)
    for i, b in enumerate(batches):
        ops = torch.from_numpy(b.ops).cuda()
        v, st = g.mixed(ops, dev(b.keys), dev(b.values))
        ov, os_ = o.mixed(b.ops, b.keys, b.values)
        np.testing.assert_array_equal(st.cpu().numpy(), os_, err_msg=f"batch {i} status")
        np.testing.assert_array_equal(host_u32(v), ov, err_msg=f"batch {i} values")
        np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv(), err_msg=f"contents after {i}")
        assert g.stats()["buckets"] == o.stats()["buckets"]
    check_layout(g, o)
    assert g.stats()["n_downsize"] > 0


def test_batch_in_parts_equals_one_batch(oracle_mod):
    """dyc_insert_begin/_part/_end (and the delete analogue) form ONE batch: one
    resize decision and one alpha check, so the statuses, contents and the resize
    schedule equal the single-batch oracle's."""
    wl = W.random_op_stream(777, n_batches=12, batch=20000, universe=40000, init_capacity=64)
    g, o = make_pair(oracle_mod, wl, B=8)
    for i, b in enumerate(wl.batches):
        n = b.keys.size
        cuts = [0, n // 3, n // 3, (2 * n) // 3, n]            # includes an empty part
        kd = dev(b.keys)
        if b.op == "insert":
            vd = dev(b.values)
            g.insert_begin(n)
            st = [g.insert_part(kd[cuts[j]:cuts[j + 1]], vd[cuts[j]:cuts[j + 1]]) for j in range(4)]
            g.insert_end()
            np.testing.assert_array_equal(torch.cat(st).cpu().numpy(), o.insert(b.keys, b.values))
        elif b.op == "delete":
            g.delete_begin(n)
            parts = [g.delete_part(kd[cuts[j]:cuts[j + 1]]) for j in range(4)]
            g.delete_end()
            ov, os_ = o.delete(b.keys)
            np.testing.assert_array_equal(torch.cat([p[1] for p in parts]).cpu().numpy(), os_)
            np.testing.assert_array_equal(host_u32(torch.cat([p[0] for p in parts])), ov)
        else:
            v, f = g.find(kd)
            ov, of = o.find(b.keys)
            np.testing.assert_array_equal(f.cpu().numpy(), of)
        np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
        assert g.stats()["buckets"] == o.stats()["buckets"], f"schedule diverged at batch {i}"


def test_lazy_delete_readback_keeps_policy_exact(oracle_mod):
    """Delete batches that cannot trigger the alpha loop (m - n >= alpha*N,
    P:L305) leave their removal count on the device; the next insert whose
    upper bound m + n crosses beta*N must apply it first, so the resize
    schedule stays the oracle's (no spurious upsize)."""
    rng = np.random.default_rng(0x1A2B)
    keys = rng.choice(np.arange(1, 1 << 30, dtype=np.uint32), size=70000, replace=False)
    vals = rng.integers(0, 1 << 31, size=keys.size, dtype=np.uint32)
    g = Table(d=4, init_capacity=1 << 16, alpha=0.3, beta=0.85, bucket_slots=8, seed=7)
    o = oracle_mod.OracleTable(d=4, init_capacity=1 << 16, alpha=0.3, beta=0.85, bucket_slots=8, seed=7)
    g.insert(dev(keys[:50000]), dev(vals[:50000]))
    o.insert(keys[:50000], vals[:50000])
    s0 = g.stats()
    for j in range(5):
        dk = keys[j * 2000:(j + 1) * 2000]
        _, st = g.delete(dev(dk))
        _, ost = o.delete(dk)
        np.testing.assert_array_equal(st.cpu().numpy(), ost)
    s1 = g.stats()
    assert s1["n_sync"] - s0["n_sync"] < 5, "delete batches still read their counters back"
    assert s1["m"] == o.stats()["m"] == 40000
    g.insert(dev(keys[50000:60000]), dev(vals[50000:60000]))
    o.insert(keys[50000:60000], vals[50000:60000])
    for j in range(5, 8):                      # lazy again, then an insert crossing beta*N
        dk = keys[j * 2000:(j + 1) * 2000]
        g.delete(dev(dk))
        o.delete(dk)
    g.insert(dev(keys[60000:70000]), dev(vals[60000:70000]))
    o.insert(keys[60000:70000], vals[60000:70000])
    gs, os_ = g.stats(), o.stats()
    assert gs["m"] == os_["m"]
    assert gs["buckets"] == os_["buckets"]
    assert gs["n_upsize"] == os_["n_upsize"]
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
    check_layout(g, o)


def test_lazy_deletes_crossing_alpha_downsize_like_oracle(oracle_mod):
    """Consecutive delete batches that together cross alpha*N, with no stats()
    or dump() in between (either would make m exact again): the skip test must
    use a lower bound of m (every pending removal subtracted), so the alpha
    loop fires in the same batch as in the oracle.  C1's eight
    delete batches back to back, then C1-like batches at a larger scale."""
    for n_keys, batch in ((65536, 8192), (200000, 10000)):
        wl = W.c1_rand_small(n_keys=n_keys, batch=batch)
        g, o = make_pair(oracle_mod, wl, B=8)
        sizes_g, sizes_o = [], []
        dels = [b for b in wl.batches if b.op == "delete"]
        ins = [b for b in wl.batches if b.op == "insert"]
        for b in ins:
            g.insert(dev(b.keys), dev(b.values))
            o.insert(b.keys, b.values)
        s0 = g.stats()
        assert s0["buckets"] == o.stats()["buckets"]
        outs = []
        for b in dels:                       # no stats/dump between the batches
            outs.append(g.delete(dev(b.keys)))
            o.delete(b.keys)
            sizes_o.append(o.stats()["buckets"])
            sizes_g.append(list(g._buckets_host()))
        for b, (v, st) in zip(dels, outs):
            assert (st.cpu().numpy() == 1).all()
            np.testing.assert_array_equal(host_u32(v), W.val_of(b.keys, 0))
        assert sizes_g == sizes_o, "downsize schedule diverged from the oracle's"
        gs, os_ = g.stats(), o.stats()
        assert gs["n_downsize"] == os_["n_downsize"] and gs["m"] == os_["m"] == 0
        assert gs["buckets"] == os_["buckets"]


def test_lazy_delete_on_other_stream_then_stats(oracle_mod):
    """A delete that skips its read-back on stream A, then stats() on stream B
    without any host wait: the read-back must wait for A's removals (event)
    before reading and resetting the device count."""
    n = 1 << 21
    keys = W.key_range(0, n, 4242)
    vals = W.val_of(keys, 0)
    g = Table(d=4, init_capacity=int(n / 0.8), alpha=0.1, beta=0.85, bucket_slots=8)
    g.insert(dev(keys), dev(vals))
    torch.cuda.synchronize()
    sa = torch.cuda.Stream()
    kd = dev(keys[: n // 4])
    torch.cuda.synchronize()
    s0 = g.stats()["n_sync"]
    with torch.cuda.stream(sa):
        g.delete(kd, stream=sa)
    s = g.stats(stream=torch.cuda.current_stream())
    assert s["n_sync"] - s0 <= 2, "the delete was expected to skip its read-back"
    assert s["m"] == n - n // 4 and sum(s["count"]) == s["m"]


def test_mixed_batch_without_host_waits_and_invalid_codes(oracle_mod):
    """dyc_mixed_batch groups its phases on the device: the phase sizes are read
    back only when the host's bound (n) cannot rule out a resize decision, so
    batches far from both fill bounds run without any host wait, and op codes
    outside 0..2 are no-ops (status NONE, value NOT_FOUND; reading Q10).
    Results equal the oracle's throughout."""
    meta, batches = W.c4_zipf_mixed(U=200000, distinct=20000, grow_batches=6, cycles=1, init_capacity=1 << 20)
    g = Table(d=4, init_capacity=1 << 20, alpha=0.01, beta=0.85, bucket_slots=8)
    o = oracle_mod.OracleTable(d=4, init_capacity=1 << 20, alpha=0.01, beta=0.85, bucket_slots=8)
    bg = W.key_range(1 << 30, 200000, 11)                 # background: far above alpha*N from here on
    g.insert(dev(bg), dev(W.val_of(bg, 0)))
    o.insert(bg, W.val_of(bg, 0))
    s0 = g.stats()
    rng = np.random.default_rng(3)
    for i, b in enumerate(batches[:8]):
        ops = b.ops.copy()
        ops[rng.choice(ops.size, size=50, replace=False)] = 7          # invalid codes
        v, st = g.mixed(torch.from_numpy(ops).cuda(), dev(b.keys), dev(b.values))
        ov, os_ = o.mixed(ops, b.keys, b.values)
        np.testing.assert_array_equal(st.cpu().numpy(), os_, err_msg=f"batch {i} status")
        np.testing.assert_array_equal(host_u32(v), ov, err_msg=f"batch {i} values")
    s1 = g.stats()
    assert s1["n_sync"] - s0["n_sync"] <= 2, s1["n_sync"] - s0["n_sync"]
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
