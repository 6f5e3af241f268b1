"""Parity of the wide-key CUDA path (include/dycuckoo_wide.h, NEXT-3) with the
wide oracle (oracle/dyw_oracle.c), in all three placement modes: per-op statuses,
find/delete values, sorted contents and subtable sizes after every batch, the
GPU layout checked with the oracle's hash (I1, I2), and the device hash against
the golden vectors written from the oracle."""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200.wide import WideTable  # noqa: E402
from tests.test_oracle_wide import E64, random_stream, wide_keys, wide_vals  # noqa: E402

MODES = [("voter", 1), ("voter", 2), ("voter", 4), ("grouped", 1), ("grouped", 2), ("grouped", 4), ("lockfree", 1)]


def dev64(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64).view(np.int64)).cuda()


def host64(t):
    return t.cpu().numpy().view(np.uint64)


@pytest.fixture(scope="module")
def wo():
    import oracle
    oracle.build_oracle_wide()
    return oracle


def pair(wo, mode, Wd, cap=2048, alpha=0.3, beta=0.85, d=4):
    g = WideTable(d=d, init_capacity=cap, alpha=alpha, beta=beta, value_words=Wd, mode=mode)
    B = 8 if mode == "lockfree" else 16
    o = wo.OracleWideTable(d=d, init_capacity=cap, alpha=alpha, beta=beta, bucket_slots=B, value_words=Wd)
    return g, o


def check_layout(g, o):
    k, v, tb, bk = g.dump()
    st = g.stats()
    assert o.check_layout(st["buckets"], k, tb, bk) == 0, "I1/I2 violated on the GPU layout"
    assert sum(st["count"]) == st["m"] == k.size


def test_wide_hash_matches_golden_vectors():
    path = os.path.join(os.path.dirname(__file__), "golden", "hash_vectors_wide.txt")
    rows = [l.split() for l in open(path) if l.strip() and not l.startswith("#")]
    keys = np.array([int(r[0]) for r in rows], dtype=np.uint64)
    g = WideTable(d=4, init_capacity=4 * 16 * 1000, value_words=1)
    x, p = g.hash_probe(dev64(keys))
    x = x.cpu().numpy().view(np.uint32)
    p = p.cpu().numpy()
    for i, r in enumerate(rows):
        assert x[i].tolist() == [int(v) for v in r[1:7]], f"key {r[0]}"
        assert p[i].tolist() == [int(r[7]), int(r[8])]


@pytest.mark.parametrize("mode,Wd", MODES)
def test_wide_random_stream_parity(wo, mode, Wd):
    g, o = pair(wo, mode, Wd)
    for i, (kind, keys, vals) in enumerate(random_stream(300 + Wd, 30, Wd)):
        kd = dev64(keys)
        if kind == "insert":
            st = g.insert(kd, dev64(vals))
            np.testing.assert_array_equal(st.cpu().numpy(), o.insert(keys, vals), err_msg=f"batch {i}")
        elif kind == "find":
            v, f = g.find(kd)
            ov, of = o.find(keys)
            np.testing.assert_array_equal(f.cpu().numpy(), of, err_msg=f"batch {i} found")
            np.testing.assert_array_equal(host64(v), ov, err_msg=f"batch {i} values")
        else:
            v, st = g.delete(kd)
            ov, os_ = o.delete(keys)
            np.testing.assert_array_equal(st.cpu().numpy(), os_, err_msg=f"batch {i} delete status")
            np.testing.assert_array_equal(host64(v), ov, err_msg=f"batch {i} old values")
        gk, gv = g.sorted_items()
        ok, ov_ = o.sorted_items()
        np.testing.assert_array_equal(gk, ok, err_msg=f"keys after batch {i}")
        np.testing.assert_array_equal(gv, ov_, err_msg=f"values after batch {i}")
        gs, os2 = g.stats(), o.stats()
        assert gs["m"] == os2["m"]
        if gs["n_fail_upsize"] == 0 and os2["n_fail_upsize"] == 0:
            assert gs["buckets"] == os2["buckets"], f"resize schedule diverged at batch {i}"
        assert gs["m"] <= 0.85 * gs["N"]
        check_layout(g, o)
    assert g.stats()["n_downsize"] > 0


@pytest.mark.parametrize("mode,Wd", [("voter", 2), ("grouped", 2), ("lockfree", 1)])
def test_wide_contended_big_batch(wo, mode, Wd):
    """One batch far larger than the table: the policy upsizes first, then every
    bucket sees ~13 concurrent placements (lock contention / CAS conflicts)."""
    g, o = pair(wo, mode, Wd, cap=64)
    k = wide_keys(0, 20000, 77)
    v = wide_vals(k, Wd, 5)
    np.testing.assert_array_equal(g.insert(dev64(k), dev64(v)).cpu().numpy(), o.insert(k, v))
    gk, gv = g.sorted_items()
    ok, ov = o.sorted_items()
    np.testing.assert_array_equal(gk, ok)
    np.testing.assert_array_equal(gv, ov)
    assert g.stats()["buckets"] == o.stats()["buckets"]
    check_layout(g, o)
    # updates of every key in one batch, then delete all: alpha loop down to one bucket
    v2 = wide_vals(k, Wd, 6)
    np.testing.assert_array_equal(g.insert(dev64(k), dev64(v2)).cpu().numpy(), o.insert(k, v2))
    gv_, gf = g.find(dev64(k))
    assert gf.cpu().numpy().all()
    np.testing.assert_array_equal(host64(gv_), v2)
    _, st = g.delete(dev64(k))
    assert st.cpu().numpy().all()
    o.delete(k)
    assert g.stats()["m"] == 0 and g.stats()["buckets"] == o.stats()["buckets"]


@pytest.mark.parametrize("mode,Wd", [("voter", 2), ("grouped", 4), ("lockfree", 1)])
def test_wide_resize_kernels(wo, mode, Wd):
    """Explicit split / merge on the wide layouts: contents kept,
    residual count = sum_b' max(0, |b'|+|b'+h|-B) from the pre-resize dump (I9)."""
    g, o = pair(wo, mode, Wd, cap=4 * 16 * 64, alpha=0.01, beta=0.95)
    B = 8 if mode == "lockfree" else 16
    k = wide_keys(0, 3000, 3)
    v = wide_vals(k, Wd, 1)
    g.insert(dev64(k), dev64(v))
    g.resize(+1)
    g.resize(+1)
    k0, v0, t0, b0 = g.dump()
    s0 = g.stats()
    h = s0["buckets"][1] // 2
    occ = np.bincount(b0[t0 == 1].astype(np.int64), minlength=2 * h)
    expect = int(np.maximum(0, occ[:h] + occ[h:] - B).sum())
    g.resize(-1)
    s1 = g.stats()
    assert s1["buckets"][1] == h and s1["n_residual"] - s0["n_residual"] == expect
    gk, gv = g.sorted_items()
    order = np.argsort(k, kind="stable")
    np.testing.assert_array_equal(gk, k[order])
    np.testing.assert_array_equal(gv, v[order])
    check_layout(g, o)


def test_wide_edge_cases(wo):
    g, o = pair(wo, "voter", 2)
    empty = dev64(np.zeros(0, np.uint64))
    g.insert(empty, dev64(np.zeros((0, 2), np.uint64)))
    keys = np.array([E64, 0xFFFFFFFF, 0, 1 << 63], dtype=np.uint64)
    vals = wide_vals(keys, 2, 0)
    np.testing.assert_array_equal(g.insert(dev64(keys), dev64(vals)).cpu().numpy(), o.insert(keys, vals))
    v, f = g.find(dev64(keys))
    ov, of = o.find(keys)
    np.testing.assert_array_equal(f.cpu().numpy(), of)
    np.testing.assert_array_equal(host64(v), ov)
    from paper_conf_icde_lizlhs21_b200._lib import DycError
    with pytest.raises(DycError):
        WideTable(value_words=2, mode="lockfree")
    with pytest.raises(DycError):
        WideTable(value_words=3)
