"""Resize under live traffic.

dyc_resize_begin runs the split/merge of one subtable on a second stream while
batches keep running on the caller's stream with that subtable locked.  The
claim pinned here: every batch issued inside the window returns exactly what the
oracle returns for the sequential order "resize, then the same batches"
(statuses, values), and after the commit the contents, the subtable sizes and
the layout (I1, I2, I4) match as well.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200._lib import DycError  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import Table  # noqa: E402

from tests.test_gpu_parity import check_layout, dev, host_u32  # noqa: E402


def _pair(oracle_mod, n, B, fill, alpha=0.05, beta=0.9):
    cap = int(n / fill)
    g = Table(d=4, init_capacity=cap, alpha=alpha, beta=beta, bucket_slots=B)
    o = oracle_mod.OracleTable(d=4, init_capacity=cap, alpha=alpha, beta=beta, bucket_slots=B)
    k = W.key_range(0, n, 41)
    v = W.val_of(k, 0)
    np.testing.assert_array_equal(g.insert(dev(k), dev(v)).cpu().numpy(), o.insert(k, v))
    return g, o, k


def _find(g, o, keys, tag):
    v, f = g.find(dev(keys))
    ov, of = o.find(keys)
    np.testing.assert_array_equal(f.cpu().numpy(), of, err_msg=f"{tag}: found")
    np.testing.assert_array_equal(host_u32(v), ov, err_msg=f"{tag}: values")


def _insert(g, o, keys, vals, tag):
    st = g.insert(dev(keys), dev(vals))
    np.testing.assert_array_equal(st.cpu().numpy(), o.insert(keys, vals), err_msg=f"{tag}: insert status")


def _delete(g, o, keys, tag):
    v, st = g.delete(dev(keys))
    ov, os_ = o.delete(keys)
    np.testing.assert_array_equal(st.cpu().numpy(), os_, err_msg=f"{tag}: delete status")
    np.testing.assert_array_equal(host_u32(v), ov, err_msg=f"{tag}: old values")


def _finish(g, o):
    g.resize_commit()
    assert g.resize_query() == (False, True)
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
    gs, os_ = g.stats(), o.stats()
    assert gs["m"] == os_["m"]
    if gs["n_fail_upsize"] == 0 and os_["n_fail_upsize"] == 0:
        assert gs["buckets"] == os_["buckets"]
    check_layout(g, o)
    return gs


@pytest.mark.parametrize("B", [4, 8])
@pytest.mark.parametrize("direction", [+1, -1])
def test_window_batches_equal_sequential_order(oracle_mod, B, direction):
    n = 40000
    g, o, k = _pair(oracle_mod, n, B, fill=0.8 if direction > 0 else 0.3)
    if direction < 0:                     # make one subtable the unique largest
        g.resize(+1)
        o.resize(+1)
    rs = torch.cuda.Stream()
    g.resize_begin(direction, resize_stream=rs)
    o.resize(direction)
    assert g.resize_query()[0]
    rng = np.random.default_rng(7 + B + direction)
    miss = W.key_range(1 << 31, 4000, 41)
    # finds never commit: the window stays open across them
    _find(g, o, np.concatenate([rng.choice(k, 4000, replace=False), miss]), "find 1")
    _find(g, o, rng.choice(k, 9000, replace=False), "find 2")
    assert g.resize_query()[0], "a find batch must not commit the resize"
    # updates of existing keys (some live in the locked subtable -> deferred) + new keys
    upd = rng.choice(k, 6000, replace=False)
    new = W.key_range(1 << 30, 3000, 41)
    ik = np.concatenate([upd, new])
    _insert(g, o, ik, W.val_of(ik, 1), "insert")
    _find(g, o, np.concatenate([upd[:2000], new[:1000], miss[:500]]), "find 3")
    dk = np.concatenate([rng.choice(np.setdiff1d(k, upd), 5000, replace=False), miss[:300]])
    _delete(g, o, dk, "delete")
    _find(g, o, np.concatenate([dk[:2000], upd[-1000:]]), "find 4")
    gs = _finish(g, o)
    assert gs["n_live_resize"] == 1
    assert gs["n_deferred"] > 0, "updates/deletes of keys in the locked subtable should have been deferred"


@pytest.mark.parametrize("direction", [+1, -1])
def test_window_without_writes_to_locked_subtable(oracle_mod, direction):
    """A window of finds plus deletes of absent keys never needs the locked
    subtable: nothing is deferred and the explicit commit installs the resize."""
    n = 30000
    g, o, k = _pair(oracle_mod, n, 8, fill=0.7 if direction > 0 else 0.3)
    if direction < 0:
        g.resize(+1)
        o.resize(+1)
    rs = torch.cuda.Stream()
    g.resize_begin(direction, resize_stream=rs)
    o.resize(direction)
    _find(g, o, k[::3], "find")
    _delete(g, o, W.key_range(1 << 31, 2000, 41), "delete misses")
    assert g.resize_query()[0]
    gs = _finish(g, o)
    assert gs["n_deferred"] == 0 and gs["n_live_resize"] == 1


def test_window_policy_commits_first(oracle_mod):
    """An insert batch that could need an upsize beyond the one in flight
    ((m+n) > beta*N_after) commits first; the schedule equals the oracle's."""
    n = 20000
    g, o, k = _pair(oracle_mod, n, 8, fill=0.84, alpha=0.2, beta=0.85)
    rs = torch.cuda.Stream()
    g.resize_begin(+1, resize_stream=rs)
    o.resize(+1)
    big = W.key_range(1 << 30, 40000, 43)
    _insert(g, o, big, W.val_of(big, 2), "big insert")
    assert not g.resize_query()[0]
    _finish(g, o)


def test_window_alpha_loop_commits_first(oracle_mod):
    """A delete batch that drops the fill below alpha of the post-resize size
    commits the downsize in flight, then runs the alpha loop."""
    n = 20000
    g, o, k = _pair(oracle_mod, n, 8, fill=0.5, alpha=0.3, beta=0.85)
    g.resize(+1)
    o.resize(+1)
    rs = torch.cuda.Stream()
    g.resize_begin(-1, resize_stream=rs)
    o.resize(-1)
    _delete(g, o, k[: int(n * 0.8)], "mass delete")
    _finish(g, o)


def test_window_mixed_and_host_batches(oracle_mod):
    n = 30000
    g, o, k = _pair(oracle_mod, n, 8, fill=0.75)
    rs = torch.cuda.Stream()
    g.resize_begin(+1, resize_stream=rs)
    o.resize(+1)
    rng = np.random.default_rng(3)
    keys = np.concatenate([rng.choice(k, 6000, replace=False), W.key_range(1 << 30, 2000, 41)])
    rng.shuffle(keys)
    ops = rng.integers(0, 3, keys.size).astype(np.uint8)
    vals = W.val_of(keys, 3)
    gv, gs = g.mixed(torch.from_numpy(ops).cuda(), dev(keys), dev(vals))
    ov, os_ = o.mixed(ops, keys, vals)
    np.testing.assert_array_equal(gs.cpu().numpy(), os_)
    np.testing.assert_array_equal(host_u32(gv), ov)
    g.resize_begin(+1, resize_stream=rs)
    o.resize(+1)
    hk = W.key_range(1 << 29, 3000, 41)
    np.testing.assert_array_equal(g.insert_host(hk, W.val_of(hk, 4)), o.insert(hk, W.val_of(hk, 4)))
    v, f = g.find_host(np.concatenate([hk, keys[:500]]))
    ov, of = o.find(np.concatenate([hk, keys[:500]]))
    np.testing.assert_array_equal(f, of)
    np.testing.assert_array_equal(v, ov)
    _finish(g, o)


def test_window_refusals_and_commit_points(oracle_mod):
    g, o, k = _pair(oracle_mod, 10000, 8, fill=0.6)
    rs = torch.cuda.Stream()
    g.resize_commit()                              # nothing in flight: no-op
    g.resize_begin(+1, resize_stream=rs)
    with pytest.raises(DycError):
        g.resize_begin(+1, resize_stream=rs)       # one resize in flight at a time
    with pytest.raises(DycError):
        g.resize_begin(+2, resize_stream=rs)
    s = g.stats()                                  # stats commits first
    assert not g.resize_query()[0] and s["n_live_resize"] == 1
    g.resize_begin(+1, resize_stream=rs)
    g.resize(+1)                                   # an explicit resize commits first
    assert not g.resize_query()[0]
    o.resize(+1)
    o.resize(+1)
    o.resize(+1)
    _finish(g, o)
    g.resize_begin(-1, resize_stream=rs)
    g.clear()
    assert g.stats()["m"] == 0
