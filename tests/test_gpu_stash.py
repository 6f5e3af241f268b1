"""Lazily settled inserts and the stash (P:L737 failure-triggered
resizing, reading Q17): an insert batch that needs no resize decision returns
without a host wait, and pairs its placement could not settle within max_hops
wait in a device stash that find, insert (existence check, update) and delete
consult until the next read-back places them.  The map semantics
must not notice: every per-op result equals the oracle's (which settles its
failures inside the batch) while the stash is populated, and the contents
after the settle equal the oracle's."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import Table  # noqa: E402
from tests.test_gpu_contention import hot_keys, check  # noqa: E402
from tests.test_gpu_parity import dev, host_u32  # noqa: E402


@pytest.mark.parametrize("B", [4, 8])
def test_stash_is_consulted_until_settled(oracle_mod, B):
    d, n0 = 4, 64
    init = d * B * n0
    g = Table(d=d, init_capacity=init, alpha=0.05, beta=0.85, bucket_slots=B, max_hops=1, seed=0xC0FFEE)
    o = oracle_mod.OracleTable(d=d, init_capacity=init, alpha=0.05, beta=0.85, bucket_slots=B, max_hops=1,
                               seed=0xC0FFEE)
    hot = hot_keys(o, n0, (0, 1), 5, 9, want=260)
    a, b = hot[:200], hot[200:250]
    # background keys first, read back exactly: from here on a lower bound of
    # m stays above alpha*N, so no batch below needs a read-back
    bg = np.setdiff1d(W.key_range(1 << 29, int(0.4 * init), 3), hot)
    g.insert(dev(bg), dev(W.val_of(bg, 0)))
    o.insert(bg, W.val_of(bg, 0))
    s0 = g.stats()

    def ins(k, ver):
        st = g.insert(dev(k), dev(W.val_of(k, ver)))
        np.testing.assert_array_equal(st.cpu().numpy(), o.insert(k, W.val_of(k, ver)))

    def fnd(k):
        v, f = g.find(dev(k))
        ov, of = o.find(k)
        np.testing.assert_array_equal(f.cpu().numpy(), of)
        np.testing.assert_array_equal(host_u32(v), ov)

    def dele(k):
        v, st = g.delete(dev(k))
        ov, ost = o.delete(k)
        np.testing.assert_array_equal(st.cpu().numpy(), ost)
        np.testing.assert_array_equal(host_u32(v), ov)

    ins(a, 0)                                   # 200 keys, 2B slots: most fail -> stash (no read-back)
    sh = g.shape()
    assert sh["m_hi"] > sh["m_lo"], "the insert was expected to skip its read-back"
    fnd(np.concatenate([a, b, W.key_range(1 << 31, 50, 1)]))     # stash hits, misses
    ins(np.concatenate([a[::3], b]), 1)         # updates of stashed keys + new hot keys
    fnd(a)
    dele(a[1::4])                                # deletes of stashed (and placed) keys
    fnd(np.concatenate([a, b]))
    ins(a[1::4][:20], 2)                        # re-insert some deleted ones
    fnd(np.concatenate([a, b]))
    sh = g.shape()
    assert sh["n_fail_upsize"] == 0, "nothing may be settled before the read-back"
    s1 = g.stats()                              # read-back: the stash is settled (failure upsizes)
    assert s1["n_fail_upsize"] > 0
    check(g, o, "after the settle")
    fnd(np.concatenate([a, b]))


def test_lazy_inserts_skip_read_backs(oracle_mod):
    """A run of inserts well below beta*N: no host wait per batch (n_sync), and
    the counts, contents and the resize schedule equal the oracle's once read."""
    n = 1 << 18
    g = Table(d=4, init_capacity=4 * n, alpha=0.01, beta=0.85, bucket_slots=8)
    o = oracle_mod.OracleTable(d=4, init_capacity=4 * n, alpha=0.01, beta=0.85, bucket_slots=8)
    keys = W.key_range(0, n, 555)
    s0 = g.stats()
    for j in range(8):
        k = keys[j * (n // 8):(j + 1) * (n // 8)]
        st = g.insert(dev(k), dev(W.val_of(k, j)))
        np.testing.assert_array_equal(st.cpu().numpy(), o.insert(k, W.val_of(k, j)))
    # the first batch reads back (a lower bound of m below alpha*N: the alpha
    # loop might fire); the next seven do not
    sh = g.shape()
    assert sh["m_lo"] == n // 8 and sh["m_hi"] == n, sh
    s1 = g.stats()
    assert s1["n_sync"] - s0["n_sync"] <= 3, s1["n_sync"] - s0["n_sync"]
    assert s1["m"] == n and s1["buckets"] == o.stats()["buckets"]
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
