"""In-place subtable resizing in reserved virtual address ranges
(DYC_RESIZE_IN_PLACE, opt-in): an upsize maps only the new half
behind the old buckets and splits there, a downsize merges into
the lower half and unmaps the upper one at the next read-back.
Here: C1 and random streams equal the oracle on this path, the physical memory
follows the table's size, and a live resize moves its subtable off the virtual
range without changing any result."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import Table  # noqa: E402
from tests.test_gpu_parity import dev  # noqa: E402

GRAN = 2 << 20


def test_c1_in_place(oracle_mod):
    """C1 (17 upsizes, 49 downsizes) on the in-place path: every batch equals
    the oracle (statuses, values, contents, resize schedule)."""
    import tests.test_gpu_parity as P
    wl = W.c1_rand_small()
    g = Table(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta, bucket_slots=8, in_place=True)
    o = oracle_mod.OracleTable(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha, beta=wl.beta, bucket_slots=8)
    for i, b in enumerate(wl.batches):
        if b.op == "insert":
            np.testing.assert_array_equal(g.insert(dev(b.keys), dev(b.values)).cpu().numpy(), o.insert(b.keys, b.values))
        elif b.op == "find":
            v, f = g.find(dev(b.keys))
            ov, of = o.find(b.keys)
            np.testing.assert_array_equal(f.cpu().numpy(), of)
            np.testing.assert_array_equal(P.host_u32(v), ov)
        else:
            v, st = g.delete(dev(b.keys))
            np.testing.assert_array_equal(st.cpu().numpy(), o.delete(b.keys)[1])
        np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
        assert g.stats()["buckets"] == o.stats()["buckets"], f"schedule diverged at batch {i}"
    s = g.stats()
    assert s["vm_subtables"] == 4
    # C1's subtables never outgrow one 2 MB granule each
    assert s["vm_mapped_bytes"] <= 4 * GRAN


def test_large_growth_and_shrink_in_place(oracle_mod):
    """2^22 keys from a 4K-slot table: every upsize maps a new chunk; deleting
    everything halves the subtables back and returns the chunks."""
    n = 1 << 22
    keys = W.key_range(0, n, 9)
    g = Table(d=4, init_capacity=4096, alpha=0.3, beta=0.85, in_place=True)
    o = oracle_mod.OracleTable(d=4, init_capacity=4096, alpha=0.3, beta=0.85, bucket_slots=8)
    for j in range(4):
        k = keys[j * (n // 4):(j + 1) * (n // 4)]
        np.testing.assert_array_equal(g.insert(dev(k), dev(W.val_of(k, 0))).cpu().numpy(),
                                      o.insert(k, W.val_of(k, 0)))
    s = g.stats()
    assert s["buckets"] == o.stats()["buckets"] and s["vm_subtables"] == 4 and s["n_vm_map"] > 4
    assert s["vm_mapped_bytes"] >= s["N"] * 8 and s["vm_mapped_bytes"] <= s["N"] * 8 + 4 * GRAN
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
    for j in range(4):
        k = keys[j * (n // 4):(j + 1) * (n // 4)]
        _, st = g.delete(dev(k))
        _, ost = o.delete(k)
        np.testing.assert_array_equal(st.cpu().numpy(), ost)
    s = g.stats()
    assert s["m"] == 0 and s["buckets"] == o.stats()["buckets"] and s["n_vm_unmap"] > 0
    assert s["vm_mapped_bytes"] <= s["N"] * 8 + 4 * GRAN


@pytest.mark.parametrize("B", [4, 8])
def test_random_streams_in_place(oracle_mod, B):
    wl = W.random_op_stream(31337 + B, n_batches=20, batch=3000, universe=6000, init_capacity=64)
    g = Table(d=4, init_capacity=64, alpha=wl.alpha, beta=wl.beta, bucket_slots=B, in_place=True)
    o = oracle_mod.OracleTable(d=4, init_capacity=64, alpha=wl.alpha, beta=wl.beta, bucket_slots=B)
    for b in wl.batches:
        if b.op == "insert":
            np.testing.assert_array_equal(g.insert(dev(b.keys), dev(b.values)).cpu().numpy(), o.insert(b.keys, b.values))
        elif b.op == "find":
            assert (g.find(dev(b.keys))[1].cpu().numpy() == o.find(b.keys)[1]).all()
        else:
            assert (g.delete(dev(b.keys))[1].cpu().numpy() == o.delete(b.keys)[1]).all()
        np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
        assert g.stats()["buckets"] == o.stats()["buckets"]
    assert g.stats()["vm_subtables"] == 4


def test_live_resize_leaves_the_virtual_range(oracle_mod):
    g = Table(d=4, init_capacity=1 << 14, alpha=0.05, beta=0.9, in_place=True)
    o = oracle_mod.OracleTable(d=4, init_capacity=1 << 14, alpha=0.05, beta=0.9, bucket_slots=8)
    k = W.key_range(0, 9000, 3)
    g.insert(dev(k), dev(W.val_of(k, 0)))
    o.insert(k, W.val_of(k, 0))
    side = torch.cuda.Stream()
    g.resize_begin(+1, resize_stream=side)
    o.resize(+1)
    v, f = g.find(dev(k))
    assert (f.cpu().numpy() == 1).all()
    g.resize_commit()
    s = g.stats()
    assert s["vm_subtables"] == 3 and s["buckets"] == o.stats()["buckets"]
    g.resize(+1)          # the smallest: one of the three still in place
    o.resize(+1)
    np.testing.assert_array_equal(g.sorted_kv(), o.sorted_kv())
    assert g.stats()["buckets"] == o.stats()["buckets"]
