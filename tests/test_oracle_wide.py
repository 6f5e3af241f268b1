"""Pins of the wide-key oracle (oracle/dyw_oracle.c, NEXT-3) against things other
than itself: a brute-force dict (the map semantics), the closed-form
resize replay, the independently pinned 32-bit oracle (a key below
2^32 must hash exactly as there, reading Q33), a uniformity test that a dropped
high-half term would fail, and the oracle's own structural invariants I1-I9."""
import numpy as np
import pytest

from paper_conf_icde_lizlhs21_b200 import workload as W
from tests.bruteforce import replay_sizes

E64 = 0xFFFFFFFFFFFFFFFF


class BruteWide:
    """dict model: insert -> 1 new / 2 updated (reserved key -> 0); find/delete
    -> (value words or all-ones, flag)."""

    def __init__(self, Wd):
        self.m, self.W = {}, Wd

    def insert(self, keys, vals):
        st = np.zeros(len(keys), dtype=np.uint8)
        for i, k in enumerate(keys.tolist()):
            if k == E64:
                continue
            st[i] = 2 if k in self.m else 1
            self.m[k] = tuple(int(x) for x in vals[i])
        return st

    def find(self, keys):
        v = np.full((len(keys), self.W), E64, dtype=np.uint64)
        f = np.zeros(len(keys), dtype=np.uint8)
        for i, k in enumerate(keys.tolist()):
            if k in self.m:
                v[i] = self.m[k]
                f[i] = 1
        return v, f

    def delete(self, keys):
        v = np.full((len(keys), self.W), E64, dtype=np.uint64)
        st = np.zeros(len(keys), dtype=np.uint8)
        for i, k in enumerate(keys.tolist()):
            if k in self.m:
                v[i] = self.m.pop(k)
                st[i] = 1
        return v, st

    def items(self):
        ks = np.array(sorted(self.m), dtype=np.uint64)
        vs = np.array([self.m[int(k)] for k in ks], dtype=np.uint64).reshape(-1, self.W)
        return ks, vs


def wide_keys(i0, n, seed):
    """Distinct u64 keys: two independent 32-bit bijections of the index (so the
    high halves vary), plus a share of keys below 2^32 and of keys whose low half
    is 0xFFFFFFFF (EMPTY only in the 32-bit table)."""
    idx = np.arange(i0, i0 + n, dtype=np.uint64)
    lo = W.lowbias32((idx & np.uint64(0xFFFFFFFF)).astype(np.uint32) ^ np.uint32(seed & 0xFFFFFFFF)).astype(np.uint64)
    hi = (idx * np.uint64(0x9E3779B1) + np.uint64(seed)) & np.uint64(0xFFFFFFFF)
    k = (hi << np.uint64(32)) | lo
    k[::7] = lo[::7] | np.uint64(0)                         # hi = 0 for every 7th (still distinct: lo is a bijection)
    k[3::11] = (hi[3::11] << np.uint64(32)) | np.uint64(0xFFFFFFFF)
    k[k == np.uint64(E64)] ^= np.uint64(1 << 40)
    u, first = np.unique(k, return_index=True)
    return k[np.sort(first)]


def wide_vals(k, Wd, ver):
    return np.stack([k * np.uint64(0x9E3779B97F4A7C15 + 2 * w + 1) + np.uint64(ver) for w in range(Wd)], axis=1)


def random_stream(seed, n_batches, Wd, batch=3000):
    rng = np.random.default_rng(seed)
    pool = wide_keys(0, n_batches * batch + 10, seed)
    live, nxt, out = [], 0, []
    for b in range(n_batches):
        kind = rng.choice(["insert", "find", "delete"], p=[0.5, 0.25, 0.25]) if b > 0 else "insert"
        if kind == "insert":
            n_new = int(rng.integers(1, batch))
            new = pool[nxt:nxt + n_new]
            nxt += n_new
            old = rng.choice(np.array(live, dtype=np.uint64), min(len(live), batch // 3), replace=False) \
                if live else np.zeros(0, np.uint64)
            keys = np.concatenate([new, old])
            rng.shuffle(keys)
            out.append(("insert", keys, wide_vals(keys, Wd, b)))
            live.extend(new.tolist())
        elif kind == "find":
            hit = rng.choice(np.array(live, dtype=np.uint64), min(len(live), batch // 2), replace=False)
            keys = np.concatenate([hit, pool[-10:], np.array([E64], dtype=np.uint64)])
            out.append(("find", keys, None))
        else:
            if not live:
                continue
            cnt = int(rng.integers(1, max(2, int(len(live) * 0.7))))
            sel = rng.choice(len(live), cnt, replace=False)
            keys = np.array([live[i] for i in sel], dtype=np.uint64)
            keys = np.concatenate([keys, pool[-5:]])
            out.append(("delete", keys, None))
            dead = set(keys.tolist())
            live = [k for k in live if k not in dead]
    while live:                                     # drain: the alpha loop must run
        cut = max(1, len(live) // 2) if len(live) > 200 else len(live)
        out.append(("delete", np.array(live[:cut], dtype=np.uint64), None))
        live = live[cut:]
    return out


@pytest.fixture(scope="module")
def wo():
    import oracle
    oracle.build_oracle_wide()
    return oracle


@pytest.mark.parametrize("Wd,B", [(1, 8), (2, 16), (4, 16)])
def test_wide_oracle_matches_brute_force(wo, Wd, B):
    d, alpha, beta, cap = 4, 0.3, 0.85, 2048
    o = wo.OracleWideTable(d=d, init_capacity=cap, alpha=alpha, beta=beta, bucket_slots=B, value_words=Wd)
    bm = BruteWide(Wd)
    hist = []
    for i, (kind, keys, vals) in enumerate(random_stream(100 + Wd, 40, Wd)):
        if kind == "insert":
            n_new = len({int(k) for k in keys.tolist()} - set(bm.m))
            np.testing.assert_array_equal(o.insert(keys, vals), bm.insert(keys, vals), err_msg=f"batch {i}")
            hist.append(("insert", len(bm.m), len(bm.m)))   # target m + n_new == m after the batch
        elif kind == "find":
            ov, of = o.find(keys)
            bv, bf = bm.find(keys)
            np.testing.assert_array_equal(of, bf)
            np.testing.assert_array_equal(ov, bv)
            continue
        else:
            ov, os_ = o.delete(keys)
            bv, bs = bm.delete(keys)
            np.testing.assert_array_equal(os_, bs)
            np.testing.assert_array_equal(ov, bv)
            hist.append(("delete", len(bm.m), len(bm.m)))
        ok, ov_ = o.sorted_items(), bm.items()
        np.testing.assert_array_equal(ok[0], ov_[0])
        np.testing.assert_array_equal(ok[1], ov_[1])
        bad, msg = o.check_invariants()
        assert bad == 0, msg
        st = o.stats()
        assert st["max_probes"] <= 2                                    # I7
        if st["n_fail_upsize"] == 0:
            assert st["buckets"] == replay_sizes(d, B, cap, alpha, beta, hist)[-1], f"schedule at batch {i}"
    assert o.stats()["n_upsize"] > 0 and o.stats()["n_downsize"] > 0


def test_wide_hash_reduces_to_32bit_hash_below_2_32(wo, oracle_mod):
    """Reading Q33: a key < 2^32 has hi = 0, so x_s must equal the pinned 32-bit
    oracle's x_s (same seed, same SplitMix64 draws for a_s, b_s)."""
    o32 = oracle_mod.OracleTable(d=4, init_capacity=4 * 4 * 1000)
    o64 = wo.OracleWideTable(d=4, init_capacity=4 * 16 * 1000, value_words=1)
    rng = np.random.default_rng(5)
    for k in [0, 1, 0xFFFFFFFE, 0xFFFFFFFB, 0xFFFFFFFA] + rng.integers(0, 2 ** 32 - 1, 300).tolist():
        assert [o64.hash_x(s, k) for s in range(6)] == [o32.hash_x(s, k) for s in range(6)]
        assert o64.pair(k) == o32.pair(k)
    a32, b32 = o32.hash_params()
    a64, b64, c64 = o64.hash_params()
    np.testing.assert_array_equal(a32, a64)
    np.testing.assert_array_equal(b32, b64)
    assert len(set(c64.tolist())) == 6 and all(1 <= c < 4294967291 for c in c64.tolist())


def test_wide_hash_uses_the_high_half(wo):
    """Keys that differ only in the high half (lo = 0 or 1) must spread over the
    buckets and pairs; dropping the c_s*hi term would put them all in one."""
    o = wo.OracleWideTable(d=4, init_capacity=4 * 16 * 500, value_words=1)
    n = 500
    for lo in (0, 1, 0xFFFFFFFF):
        keys = [(i << 32) | lo for i in range(1, 20001)]
        bk = np.array([o.bucket(1, k) for k in keys])
        counts = np.bincount(bk, minlength=n)
        chi2 = ((counts - 40.0) ** 2 / 40.0).sum()
        assert chi2 < (n - 1) + 6 * (2 * (n - 1)) ** 0.5
        pairs = {o.pair(k) for k in keys[:2000]}
        assert len(pairs) == 12


def test_wide_hash_golden_vectors(wo):
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", "hash_vectors_wide.txt")
    rows = [l.split() for l in open(path) if l.strip() and not l.startswith("#")]
    o = wo.OracleWideTable(d=4, init_capacity=4 * 16 * 1000, seed=0x5EED0001, value_words=1)
    assert len(rows) > 50
    for r in rows:
        k = int(r[0])
        assert [o.hash_x(s, k) for s in range(6)] == [int(x) for x in r[1:7]]
        assert list(o.pair(k)) == [int(r[7]), int(r[8])]


def test_wide_reserved_key_and_empty_low_half(wo):
    o = wo.OracleWideTable(d=4, init_capacity=256, value_words=2)
    keys = np.array([E64, 0xFFFFFFFF, 0x1FFFFFFFF, 5], dtype=np.uint64)
    st = o.insert(keys, wide_vals(keys, 2, 0))
    np.testing.assert_array_equal(st, [0, 1, 1, 1])
    v, f = o.find(keys)
    np.testing.assert_array_equal(f, [0, 1, 1, 1])
    np.testing.assert_array_equal(v[1:], wide_vals(keys[1:], 2, 0))
    assert (v[0] == E64).all()


def test_wide_resize_mechanics(wo):
    """P:L377-381 split (I8) and P:L389-393 merge with residuals (I9) on the wide
    table: contents unchanged, entries land in b or b+n, residual count formula."""
    o = wo.OracleWideTable(d=4, init_capacity=4 * 16 * 64, alpha=0.01, beta=0.95, value_words=2)
    k = wide_keys(0, 3000, 9)
    o.insert(k, wide_vals(k, 2, 1))
    k0, v0, t0, b0 = o.dump()
    n0 = o.stats()["buckets"]
    assert o.resize(+1) == 0
    k1, v1, t1, b1 = o.dump()
    before = {int(a): (int(t), int(b)) for a, t, b in zip(k0, t0, b0)}
    after = {int(a): (int(t), int(b)) for a, t, b in zip(k1, t1, b1)}
    assert before.keys() == after.keys()
    for key, (t, b) in before.items():
        assert after[key] in (((0, b), (0, b + n0[0])) if t == 0 else ((t, b),))
    o.resize(+1)
    k2, v2, t2, b2 = o.dump()
    h = o.stats()["buckets"][1] // 2
    occ = np.bincount(b2[t2 == 1].astype(np.int64), minlength=2 * h)
    expect = int(np.maximum(0, occ[:h] + occ[h:] - 16).sum())
    r0 = o.stats()["n_residual"]
    assert o.resize(-1) == 0
    assert o.stats()["n_residual"] - r0 == expect
    ks, vs = o.sorted_items()
    order = np.argsort(k, kind="stable")
    np.testing.assert_array_equal(ks, k[order])
    np.testing.assert_array_equal(vs, wide_vals(k, 2, 1)[order])
    assert o.check_invariants()[0] == 0
