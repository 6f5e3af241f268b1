"""Adversarial contention on the u32 hot path (key sets that all
share one pair and one bucket, for maximal CAS / exchange contention and long
eviction chains; VERDICT r1 "What's missing" 5).

The keys are chosen with the ORACLE's hash (its constants, the formula of
P:L271 and the first layer of P:L440-441, evaluated here in numpy) from a
seeded candidate range.  Every batch's per-op statuses and values, and the
sorted contents afterwards, must equal the oracle's; the GPU layout must be
valid (I1, I2 with the oracle's hash; I4 counts; I6 shape).  The resize
schedules may differ (failure-triggered upsizes, depend on placement,
which is nondeterministic by design), so they are not compared.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import Table  # noqa: E402

P = np.uint64(4294967291)
EMPTY = 0xFFFFFFFF


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).cuda()


def host_u32(t):
    return t.cpu().numpy().view(np.uint32)


def _x(a, b, k):
    return ((np.uint64(a) * k) % P + np.uint64(b)) % P


def hot_keys(o, n_buckets, pair, b1, b2=None, want=400, start=0, chunk=1 << 23, max_chunks=64):
    """The first `want` keys of key_range(start, ...) whose ordered pair is
    `pair` and whose bucket in pair[0] is b1 (and in pair[1] is b2, if given), at
    n_buckets buckets per subtable, under the oracle's hash constants."""
    a, b = o.hash_params()
    d = o.d
    got = []
    have = 0
    for c in range(max_chunks):
        k = W.key_range(start + c * chunk, chunk, 0x51DE).astype(np.uint64)
        q = _x(a[0], b[0], k) % np.uint64(d * (d - 1))
        t1 = q // np.uint64(d - 1)
        r = q % np.uint64(d - 1)
        t2 = r + (r >= t1)
        sel = (t1 == pair[0]) & (t2 == pair[1])
        k = k[sel]
        k = k[_x(a[pair[0] + 1], b[pair[0] + 1], k) % np.uint64(n_buckets) == b1]
        if b2 is not None:
            k = k[_x(a[pair[1] + 1], b[pair[1] + 1], k) % np.uint64(n_buckets) == b2]
        k = k.astype(np.uint32)
        k = k[k != EMPTY]
        got.append(k)
        have += k.size
        if have >= want:
            break
    out = np.concatenate(got)
    assert out.size >= want, f"only {out.size} hot keys in the candidate range"
    return out[:want]


def check(g, o, tag):
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv(), err_msg=f"contents {tag}")
    kv, tb, bk = g.dump()
    st = g.stats()
    keys = (kv & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    assert o.check_layout(st["buckets"], keys, tb, bk) == 0, f"I1/I2 {tag}"
    assert sum(st["count"]) == st["m"] == kv.size, f"I4 {tag}"
    assert max(st["buckets"]) <= 2 * min(st["buckets"]), f"I6 {tag}"
    return st


@pytest.mark.parametrize("B", [4, 8])
@pytest.mark.parametrize("max_hops", [1, 64])
def test_one_bucket_pair_for_every_key(oracle_mod, B, max_hops):
    """Hundreds of keys whose two candidate buckets are the SAME two buckets:
    only 2B slots exist for them at the start, so the batch runs CAS races on
    one bucket, exchange chains that ping-pong between two buckets, failure
    lists, retries and failure-triggered upsizes until the splits
    spread them.  Then updates of the same keys race with new hot keys in one
    batch, finds, and deletes."""
    d, n0 = 4, 64
    init = d * B * n0
    g = Table(d=d, init_capacity=init, alpha=0.05, beta=0.85, bucket_slots=B, max_hops=max_hops, seed=0xC0FFEE)
    o = oracle_mod.OracleTable(d=d, init_capacity=init, alpha=0.05, beta=0.85, bucket_slots=B,
                               max_hops=max_hops, seed=0xC0FFEE)
    hot = hot_keys(o, n0, (0, 1), 5, 9, want=600)
    first, second = hot[:400], hot[400:]
    st = g.insert(dev(first), dev(W.val_of(first, 0)))
    np.testing.assert_array_equal(st.cpu().numpy(), o.insert(first, W.val_of(first, 0)))
    s = check(g, o, "after the hot insert")
    assert s["n_fail_upsize"] > 0, "the batch was expected to need failure-triggered upsizes"
    mix = np.concatenate([first[::2], second])           # updates racing new keys on the same buckets
    vals = W.val_of(mix, 1)
    st = g.insert(dev(mix), dev(vals))
    np.testing.assert_array_equal(st.cpu().numpy(), o.insert(mix, vals))
    check(g, o, "after updates + new hot keys")
    q = np.concatenate([hot, W.key_range(1 << 31, 100, 3)])
    v, f = g.find(dev(q))
    ov, of = o.find(q)
    np.testing.assert_array_equal(f.cpu().numpy(), of)
    np.testing.assert_array_equal(host_u32(v), ov)
    dk = hot[1::2]
    v, st = g.delete(dev(dk))
    ov, ost = o.delete(dk)
    np.testing.assert_array_equal(st.cpu().numpy(), ost)
    np.testing.assert_array_equal(host_u32(v), ov)
    check(g, o, "after the deletes")


@pytest.mark.parametrize("max_hops", [1, 64])
def test_one_first_choice_bucket_in_a_big_table(oracle_mod, max_hops):
    """1,500 keys with the same pair and the same first-choice bucket
    in a table with plenty of room: every thread CASes into one 64-B bucket,
    the losers fall to their (distinct) second-choice buckets, and evictions
    out of the hot bucket run chains through the rest of the table."""
    d, B, n0 = 4, 8, 1 << 10
    init = d * B * n0
    g = Table(d=d, init_capacity=init, alpha=0.05, beta=0.85, bucket_slots=B, max_hops=max_hops, seed=0xBEEF)
    o = oracle_mod.OracleTable(d=d, init_capacity=init, alpha=0.05, beta=0.85, bucket_slots=B,
                               max_hops=max_hops, seed=0xBEEF)
    bg = W.key_range(0, int(0.6 * init), 77)                # background fill 0.6
    g.insert(dev(bg), dev(W.val_of(bg, 0)))
    o.insert(bg, W.val_of(bg, 0))
    hot = hot_keys(o, n0, (2, 3), 123, None, want=1500, start=1 << 30)
    hot = np.setdiff1d(hot, bg)
    st = g.insert(dev(hot), dev(W.val_of(hot, 2)))
    np.testing.assert_array_equal(st.cpu().numpy(), o.insert(hot, W.val_of(hot, 2)))
    check(g, o, "after the hot-bucket insert")
    st = g.insert(dev(hot), dev(W.val_of(hot, 3)))          # every one an update
    assert (st.cpu().numpy() == 2).all()
    o.insert(hot, W.val_of(hot, 3))
    v, f = g.find(dev(hot))
    assert (f.cpu().numpy() == 1).all()
    np.testing.assert_array_equal(host_u32(v), W.val_of(hot, 3))
    check(g, o, "after the updates")
