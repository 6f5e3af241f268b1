"""Pins the oracle's structural layer (hashing, resize mechanics, resize policy,
eviction rule) against the paper's closed forms, worked examples and
properties that a plausible mistake would break.  No GPU needed."""
import numpy as np
import pytest

from paper_conf_icde_lizlhs21_b200 import workload as W
from tests.bruteforce import BruteMap, replay_sizes

P = 4294967291


# --------------------------------------------------------------------- hashing
def test_hash_spec_properties(oracle_mod):
    """Universal hash of P:L271 (reading Q1): x_s(k) in [0,p); for fixed s the map
    k -> x_s(k) is injective on k < p (a_s != 0 mod p); buckets cover [0,n)
    uniformly; the first layer (Q2) yields ordered pairs t1 != t2 with
    all d(d-1) pairs about equally likely."""
    d = 4
    o = oracle_mod.OracleTable(d=d, init_capacity=4 * 4 * 1000)
    a, b = o.hash_params()
    assert all(1 <= int(x) < P for x in a) and all(0 <= int(x) < P for x in b)
    assert len(set(a.tolist())) == d + 2
    keys = W.key_range(0, 20000, 12345)
    xs = [o.hash_x(1, int(k)) for k in keys]
    assert max(xs) < P and len(set(xs)) == len(xs)
    pairs = {}
    for k in keys[:12000]:
        t1, t2 = o.pair(int(k))
        assert t1 != t2 and 0 <= t1 < d and 0 <= t2 < d
        pairs[(t1, t2)] = pairs.get((t1, t2), 0) + 1
    assert len(pairs) == d * (d - 1)
    exp = 12000 / (d * (d - 1))
    assert all(abs(c - exp) < 5 * exp ** 0.5 for c in pairs.values())
    bk = np.array([o.bucket(2, int(k)) for k in keys])
    assert bk.min() >= 0 and bk.max() < 1000
    counts = np.bincount(bk, minlength=1000)
    chi2 = ((counts - 20.0) ** 2 / 20.0).sum()
    assert chi2 < 1000 + 5 * (2 * 1000) ** 0.5   # 999 dof


def test_hash_matches_golden_vectors(oracle_mod):
    """tests/golden/hash_vectors.txt was written by tests/golden/make_hash_vectors.py
    (calls only oracle/); the CUDA side is checked against the same file."""
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", "hash_vectors.txt")
    rows = [l.split() for l in open(path) if l.strip() and not l.startswith("#")]
    hdr = {}
    for l in open(path):
        if l.startswith("# seed"):
            hdr["seed"] = int(l.split()[2], 0)
    o = oracle_mod.OracleTable(d=4, init_capacity=4 * 4 * 1000, seed=hdr["seed"])
    for r in rows:
        k = int(r[0])
        assert [o.hash_x(s, k) for s in range(6)] == [int(x) for x in r[1:7]]
        assert list(o.pair(k)) == [int(r[7]), int(r[8])]


# --------------------------------------------------------------------- resize mechanics
def _filled(oracle_mod, d=4, B=4, per=64, n_keys=600, seed=7):
    o = oracle_mod.OracleTable(d=d, init_capacity=d * B * per, alpha=0.01, beta=0.95,
                               bucket_slots=B)
    k = W.key_range(0, n_keys, seed)
    o.insert(k, W.val_of(k, 0))
    return o, k


def test_upsize_split_property(oracle_mod):
    """after doubling h^t an entry of bucket loc is in loc or
    loc+|h^t|; nothing else moves; contents are unchanged (I8)."""
    o, _ = _filled(oracle_mod)
    kv0, tb0, bk0 = o.dump()
    n0 = o.stats()["buckets"]
    assert o.resize(+1) == 0
    kv1, tb1, bk1 = o.dump()
    n1 = o.stats()["buckets"]
    t = [i for i in range(4) if n1[i] != n0[i]]
    assert t == [0] and n1[0] == 2 * n0[0]          # smallest, ties -> lowest (Q12)
    before = {int(x & 0xFFFFFFFF): (int(a), int(b)) for x, a, b in zip(kv0, tb0, bk0)}
    after = {int(x & 0xFFFFFFFF): (int(a), int(b)) for x, a, b in zip(kv1, tb1, bk1)}
    assert before.keys() == after.keys()
    for k, (tt, b) in before.items():
        ta, ba = after[k]
        assert ta == tt
        if tt == 0:
            assert ba in (b, b + n0[0])
        else:
            assert ba == b
    np.testing.assert_array_equal(np.sort(kv0), np.sort(kv1))


def test_downsize_residual_count(oracle_mod):
    """merging loc and loc+|h|/2 keeps at most B per bucket; the
    residual count equals sum_b' max(0, |b'|+|b'+h| - B), computed here from the
    pre-resize dump; residuals land in their pair's other table (never t)."""
    B = 2
    o = oracle_mod.OracleTable(d=4, init_capacity=4 * B * 64, alpha=0.01, beta=0.95,
                               bucket_slots=B)
    assert o.resize(+1) == 0 and o.resize(+1) == 0   # tables 0,1 at 128 buckets
    keys = W.key_range(0, 500, 7)                    # N = 768 slots, 640 after
    o.insert(keys, W.val_of(keys, 0))
    kv0, tb0, bk0 = o.dump()
    s0 = o.stats()
    t = 1                                             # largest, ties -> highest (Q12)
    h = s0["buckets"][t] // 2
    occ = np.bincount(bk0[tb0 == t].astype(np.int64), minlength=2 * h)
    expect = int(np.maximum(0, occ[:h] + occ[h:] - B).sum())
    assert expect > 0
    assert o.resize(-1) == 0
    s1 = o.stats()
    assert s1["buckets"][t] == h and s1["n_residual"] - s0["n_residual"] == expect
    np.testing.assert_array_equal(np.sort(kv0), np.sort(o.dump()[0]))
    assert o.check_invariants()[0] == 0


@pytest.mark.parametrize("d", [2, 3, 4, 6, 8])
@pytest.mark.parametrize("d_big", [0, 1, 2])
def test_fill_after_upsize_closed_form(oracle_mod, d, d_big):
    """with d' tables of size 2n and d-d' of size n, one upsize turns
    θ into θ(d+d')/(d+d'+1), which is ≥ βd/(d+1) when θ > β."""
    if d_big >= d:
        return
    B, per, beta = 4, 32, 0.85
    o = oracle_mod.OracleTable(d=d, init_capacity=d * B * per, alpha=0.01, beta=0.99,
                               bucket_slots=B)
    for _ in range(d_big):
        assert o.resize(+1) == 0
    N = o.stats()["N"]
    assert N == B * per * (d + d_big)
    k = W.key_range(0, int(0.86 * N), 99 + d)
    o.insert(k, W.val_of(k, 0))
    s = o.stats()
    theta = s["m"] / s["N"]
    assert theta > beta
    assert o.resize(+1) == 0
    s2 = o.stats()
    assert s2["m"] == s["m"]
    theta2 = s2["m"] / s2["N"]
    assert theta2 == pytest.approx(theta * (d + d_big) / (d + d_big + 1), rel=1e-12)
    assert theta2 >= beta * d / (d + 1)


def test_resize_refuses_breaking_double_bound(oracle_mod):
    """P:L312 "no subtable will be more than double the size as others"."""
    o = oracle_mod.OracleTable(d=4, init_capacity=4 * 4 * 8)
    assert o.resize(+1, 0) == 0
    assert o.resize(+1, 0) == -1        # 0 is no longer a smallest
    assert o.resize(-1, 3) == -1        # 3 is not a largest
    assert o.resize(-1, 0) == 0


def test_c1_resize_schedule_replay(oracle_mod):
    """Config C1 subtable sizes after every batch equal an independent replay of
    the policy of P:L305-312 from the live-key count alone (Q11-Q13).
    Appendix A.1 records the same schedule: 17 upsizes, 49 downsizes, final
    1 bucket per subtable."""
    wl = W.c1_rand_small()
    o = oracle_mod.OracleTable(d=4, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta)
    bm = BruteMap()
    sizes, plan = [], []
    for b in wl.batches:
        if b.op == "insert":
            m0 = len(bm.m)
            n_new = len({int(k) for k in b.keys} - set(bm.m))
            o.insert(b.keys, b.values)
            bm.insert(b.keys, b.values)
            plan.append(("insert", m0 + n_new, len(bm.m)))
        elif b.op == "find":
            o.find(b.keys)
            plan.append(("find", len(bm.m), len(bm.m)))
        else:
            o.delete(b.keys)
            bm.delete(b.keys)
            plan.append(("delete", len(bm.m), len(bm.m)))
        sizes.append(o.stats()["buckets"])
    # find batches never resize: the replay skips the alpha loop for them
    rs = replay_sizes(4, 4, wl.init_capacity, wl.alpha, wl.beta,
                      [(k, t, m) if k != "find" else ("find", -1, 10 ** 12) for (k, t, m) in plan])
    assert sizes == rs
    s = o.stats()
    assert s["n_fail_upsize"] == 0
    assert (s["n_upsize"], s["n_downsize"]) == (17, 49)
    assert s["buckets"] == [1, 1, 1, 1]


# --------------------------------------------------------------------- worked examples
def _find_key(o, cond, start=0, limit=2_000_000, seed=4242):
    for i in range(start, limit):
        k = int(W.key_range(i, 1, seed)[0])
        if cond(k):
            return k, i + 1
    raise AssertionError("no key found")


def test_example1_eviction_goes_to_victims_partner(oracle_mod):
    """Example 1: (k,v) hashes to (h_i,h_j) and tries h_i; its bucket
    is full, so (k',v') is evicted; k' hashes to (h_i,h_t), hence it is
    re-inserted into h_t."""
    d, B, per = 4, 1, 4
    o = oracle_mod.OracleTable(d=d, init_capacity=d * B * per, bucket_slots=B, alpha=0.01, beta=0.99)
    k, nxt = _find_key(o, lambda x: True)
    i, j = o.pair(k)
    bi, bj = o.bucket(i, k), o.bucket(j, k)

    def victim_ok(x):
        if x == k:
            return False
        p = o.pair(x)
        if i not in p or o.bucket(i, x) != bi:
            return False
        t = p[1] if p[0] == i else p[0]
        return t != j
    kp, nxt = _find_key(o, victim_ok, nxt)
    tp = [t for t in o.pair(kp) if t != i][0]
    filler, nxt = _find_key(o, lambda x: x not in (k, kp) and j in o.pair(x)
                            and o.bucket(j, x) == bj, nxt)
    o.poke(i, bi, 0, kp, 111)
    o.poke(j, bj, 0, filler, 222)
    assert o.peek(tp, o.bucket(tp, kp), 0)[0] == 0xFFFFFFFF
    ev0 = o.stats()["n_evict"]
    assert o.place_one(k, 333) == 0
    assert o.peek(i, bi, 0) == (k, 333)                  # k took h_i
    assert o.peek(tp, o.bucket(tp, kp), 0) == (kp, 111)  # k' went to h_t
    assert o.peek(j, bj, 0) == (filler, 222)             # h_j untouched
    assert o.stats()["n_evict"] - ev0 == 1


def test_example2_three_inserts(oracle_mod):
    """Example 2: k1 goes into free bucket x; k33 already lives in
    bucket y and is updated; k65 finds bucket y full and evicts k64, which moves
    to a free bucket z.  Every key ends present exactly once with its latest value."""
    d, B, per = 4, 2, 8
    o = oracle_mod.OracleTable(d=d, init_capacity=d * B * per, bucket_slots=B, alpha=0.01, beta=0.99)
    k65, nxt = _find_key(o, lambda x: True)
    i, j = o.pair(k65)
    by = o.bucket(i, k65)
    k33, nxt = _find_key(o, lambda x: x != k65 and o.pair(x)[0] == i and o.bucket(i, x) == by, nxt)
    k64, nxt = _find_key(o, lambda x: x not in (k65, k33) and i in o.pair(x)
                         and o.bucket(i, x) == by
                         and [t for t in o.pair(x) if t != i][0] != j, nxt)
    bj = o.bucket(j, k65)
    f1, nxt = _find_key(o, lambda x: x not in (k65, k33, k64) and j in o.pair(x) and o.bucket(j, x) == bj, nxt)
    f2, nxt = _find_key(o, lambda x: x not in (k65, k33, k64, f1) and j in o.pair(x) and o.bucket(j, x) == bj, nxt)
    k1, nxt = _find_key(o, lambda x: x not in (k65, k33, k64, f1, f2)
                        and by != o.bucket(o.pair(x)[0], x), nxt)
    o.poke(i, by, 0, k33, 33)
    o.poke(i, by, 1, k64, 64)
    o.poke(j, bj, 0, f1, 1001)
    o.poke(j, bj, 1, f2, 1002)
    keys = np.array([k1, k33, k65], dtype=np.uint32)
    st = o.insert(keys, np.array([1, 3333, 65], dtype=np.uint32))
    assert st.tolist() == [1, 2, 1]
    c = o.contents()
    assert c == {k1: 1, k33: 3333, k65: 65, k64: 64, f1: 1001, f2: 1002}
    assert o.check_invariants()[0] == 0
    assert o.stats()["n_evict"] >= 1
