"""The first-choice-full invariant (FFI; not in the paper).

While bit t of dyc_clean_mask is set, every stored key whose first-choice
subtable is t but which lives in its second choice has a FULL bucket h_t(k).
k_find and k_upsert then skip the second probe after a miss in a non-full
first-choice bucket of t.  These tests check (1) that the invariant really holds
in the GPU layout whenever the mask claims it, after every kind of mutation,
(2) that the results stay bit-exact with the oracle across the transitions that
must clear the mask (deletes, upsizes), and (3) that the shortcut is taken.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import Table  # noqa: E402

from .test_gpu_parity import check_layout, dev, host_u32  # noqa: E402


def ffi_violations(g, B):
    """Per subtable t: number of keys with first choice t stored in their second
    choice whose bucket h_t(k) is not full (computed from the dump)."""
    kv, tb, bk = g.dump()
    st = g.stats()
    keys = (kv & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    if keys.size == 0:
        return [0] * g.d
    x, pr = g.hash_probe(dev(keys))
    x = x.cpu().numpy().view(np.uint32).astype(np.uint64)
    pr = pr.cpu().numpy()
    fill = {}
    for t, b in zip(tb.tolist(), bk.tolist()):
        fill[(t, b)] = fill.get((t, b), 0) + 1
    bad = [0] * g.d
    for j in range(keys.size):
        t1, t2 = int(pr[j, 0]), int(pr[j, 1])
        if int(tb[j]) != t2:
            continue
        b1 = int(x[j, t1 + 1] % np.uint64(st["buckets"][t1]))
        if fill.get((t1, b1), 0) < B:
            bad[t1] += 1
    return bad


def assert_mask_truthful(g, B):
    mask = g.clean_mask()
    bad = ffi_violations(g, B)
    for t in range(g.d):
        if (mask >> t) & 1:
            assert bad[t] == 0, f"mask claims FFI for subtable {t} but {bad[t]} keys violate it"
    return mask, bad


def pair(oracle_mod, n, B, alpha=0.05, beta=0.95, cap_factor=0.9):
    per = 2 * -(-int(n / cap_factor) // (2 * 4 * B))      # even bucket count per subtable (halvable)
    cap = per * 4 * B
    g = Table(d=4, init_capacity=cap, alpha=alpha, beta=beta, bucket_slots=B)
    o = oracle_mod.OracleTable(d=4, init_capacity=cap, alpha=alpha, beta=beta, bucket_slots=B)
    return g, o


def ins(g, o, k, ver):
    v = W.val_of(k, ver)
    st = g.insert(dev(k), dev(v)).cpu().numpy()
    np.testing.assert_array_equal(st, o.insert(k, v))


def fnd(g, o, k):
    v, f = g.find(dev(k))
    ov, of = o.find(k)
    np.testing.assert_array_equal(f.cpu().numpy(), of)
    np.testing.assert_array_equal(host_u32(v), ov)


def dele(g, o, k):
    v, st = g.delete(dev(k))
    ov, os_ = o.delete(k)
    np.testing.assert_array_equal(st.cpu().numpy(), os_)
    np.testing.assert_array_equal(host_u32(v), ov)


@pytest.mark.parametrize("B", [4, 8, 16])
def test_ffi_holds_after_inserts_and_is_cleared_by_deletes(oracle_mod, B):
    n = 40000
    g, o = pair(oracle_mod, n, B)
    full = (1 << g.d) - 1
    assert g.clean_mask() == full
    k = W.key_range(0, n, 7)
    ins(g, o, k, 0)                              # fill ~0.9: many keys in their second choice
    mask, bad = assert_mask_truthful(g, B)
    assert mask == full and g.stats()["n_upsize"] == 0
    ins(g, o, k, 1)                              # every key present: all UPDATED (t2 keys too)
    miss = W.key_range(1 << 31, n, 7)
    fnd(g, o, np.concatenate([k, miss]))
    # delete 30 %: buckets become non-full under keys living in their second choice
    dele(g, o, k[: n * 3 // 10])
    mask, bad = assert_mask_truthful(g, B)
    assert mask == 0
    assert sum(bad) > 0, "the workload should create FFI violations after deletes"
    ins(g, o, k, 2)                              # 70 % UPDATED (some in t2 under non-full t1), 30 % INSERTED
    fnd(g, o, np.concatenate([k, miss]))
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
    check_layout(g, o)
    g.clear()
    o2 = oracle_mod.OracleTable(d=4, init_capacity=g.stats()["N"], alpha=0.05, beta=0.95, bucket_slots=B)
    assert g.clean_mask() == full
    ins(g, o2, k, 3)
    assert_mask_truthful(g, B)


@pytest.mark.parametrize("B", [4, 8])
def test_ffi_upsize_clears_only_that_subtable_and_downsize_keeps_it(oracle_mod, B):
    n = 40000
    g, o = pair(oracle_mod, n, B, cap_factor=0.6)    # 0.6 -> 0.69 after one halving
    full = (1 << g.d) - 1
    k = W.key_range(0, n, 11)
    ins(g, o, k, 0)
    # downsize the largest (ties -> highest index, Q12): merged buckets stay full
    g.resize(-1)
    o.resize(-1)
    mask, _ = assert_mask_truthful(g, B)
    assert mask == full
    ins(g, o, k, 1)
    fnd(g, o, np.concatenate([k, W.key_range(1 << 31, n, 11)]))
    # upsize the smallest: split buckets are no longer full
    ti = int(np.argmin(g.stats()["buckets"]))
    g.resize(+1)
    o.resize(+1)
    mask, bad = assert_mask_truthful(g, B)
    assert mask == full & ~(1 << ti)
    assert bad[ti] > 0, "the split should leave keys in t2 under non-full first-choice buckets"
    ins(g, o, k, 2)                              # all UPDATED, including the ones the split exposed
    fnd(g, o, np.concatenate([k, W.key_range(1 << 31, n, 11)]))
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
    check_layout(g, o)


def test_ffi_shortcut_is_taken(oracle_mod):
    """Probe accounting: after a fresh fill, misses in non-full first-choice buckets
    skip the second probe; after deletes, every miss probes twice."""
    n, B = 1 << 16, 8
    g, o = pair(oracle_mod, n, B, cap_factor=0.8)
    k = W.key_range(0, n, 5)
    g.probe_count(True)
    ins(g, o, k, 0)
    pc = g.probe_count_read()
    ops, p2 = pc["upsert"]
    assert ops == n and p2 < 0.5 * n           # most new keys saw a non-full first-choice bucket
    miss = W.key_range(1 << 31, n, 5)
    fnd(g, o, miss)
    ops, p2 = g.probe_count_read()["find"]
    assert ops == n and 0 < p2 < n
    dele(g, o, k[: n // 4])
    g.probe_count_read()
    fnd(g, o, miss)
    ops, p2 = g.probe_count_read()["find"]
    assert (ops, p2) == (n, n)                   # mask cleared: no shortcut
    g.probe_count(False)


def test_ffi_random_streams_mask_truthful(oracle_mod):
    """Mixed random stream with resizes both ways: parity every batch, and the mask
    never claims the invariant where the layout violates it."""
    wl = W.random_op_stream(777, n_batches=24, batch=3000, universe=6000, d=4, alpha=0.3, beta=0.85,
                            init_capacity=64)
    B = 8
    g = Table(d=4, init_capacity=64, alpha=0.3, beta=0.85, bucket_slots=B)
    o = oracle_mod.OracleTable(d=4, init_capacity=64, alpha=0.3, beta=0.85, bucket_slots=B)
    for b in wl.batches:
        if b.op == "insert":
            ins_v = b.values
            st = g.insert(dev(b.keys), dev(ins_v)).cpu().numpy()
            np.testing.assert_array_equal(st, o.insert(b.keys, ins_v))
        elif b.op == "find":
            fnd(g, o, b.keys)
        else:
            dele(g, o, b.keys)
        np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
        assert_mask_truthful(g, B)
