"""Parity of the region-binned execution path (dyc_binned.cuh, dyc_set_binning)
with the CPU oracle.

Binned mode reorders the work of a batch (ops grouped by the region of the
bucket each pass probes, results written back through op-index groups); the
per-op results, the contents after every batch and the resize schedule must be
exactly those of the oracle, as for the direct kernels.  Tiny regions and result
groups (2^1 .. 2^6 buckets, 2^1 .. 2^10 ops) force many bins, bins spanning
subtable boundaries, the 1024-bin cap and ragged tails at oracle-friendly sizes.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import workload as W  # noqa: E402
from paper_conf_icde_lizlhs21_b200.table import Table  # noqa: E402

from .test_gpu_parity import EMPTY, check_layout, dev, host_u32, run_parity  # noqa: E402


@pytest.mark.parametrize("log2_n,extra,binning", [(16, 0, (1, 6, 10)), (16, 0, (1, 1, 1)),
                                                  (20, 12345, (1, 8, 14)), (20, 777, (1, 0, 0))])
def test_binned_c2_shape_parity(oracle_mod, log2_n, extra, binning):
    """C2's shape (fill to 0.85 in one insert batch, 50%-hit finds, deletes) run
    binned; ragged tails from `extra` keys beyond a power of two."""
    wl = W.c2_rand_static(log2_n=log2_n)
    if extra:
        more = W.key_range(1 << 30, extra, 99)
        b0 = wl.batches[0]
        b0.keys = np.concatenate([b0.keys, more])
        b0.values = np.concatenate([b0.values, W.val_of(more, 0)])
    g, o = run_parity(oracle_mod, wl, B=8, layout_every=(log2_n <= 16), binning=binning)
    check_layout(g, o)
    # the extra keys push (m+n) past beta*N: that insert needs an upsize first and
    # takes the direct kernels; find and delete still run binned
    assert g.binning_info()[0] == (2 if extra else 3)


@pytest.mark.parametrize("B", [4, 8, 16, 32])
@pytest.mark.parametrize("d", [2, 4, 7])
def test_binned_random_streams_parity(oracle_mod, B, d):
    """Random single-type batches with resizes in both directions: inserts that
    need an upsize take the direct kernels, all others run binned."""
    alpha = round(min(0.3, 0.85 * d / (d + 1) - 0.01), 3)
    wl = W.random_op_stream(2000 + 10 * d + B, n_batches=30, batch=3000, universe=6000, d=d,
                            alpha=alpha, beta=0.85, init_capacity=64)
    g, _ = run_parity(oracle_mod, wl, B=B, binning=(1, 3, 7))
    assert g.binning_info()[0] > 10


def test_binned_failure_path(oracle_mod):
    """max_hops = 1: pending keys of the binned placement passes hit the failure
    list and failure-triggered upsizes; nothing is lost or duplicated."""
    wl = W.random_op_stream(4343, n_batches=20, batch=4000, universe=8000, init_capacity=16)
    g, _ = run_parity(oracle_mod, wl, B=4, max_hops=1, compare_sizes=False, binning=(1, 2, 5))
    assert g.binning_info()[0] > 0


def test_binned_edge_cases(oracle_mod):
    """Reserved keys (status NONE, value NOT_FOUND), updates, misses, single-op
    and empty batches in binned mode."""
    wl = W.Workload("edge", 4, 0.3, 0.85, 4096)
    e = np.zeros(0, dtype=np.uint32)
    ks = np.array([EMPTY, 1, 2, 3], dtype=np.uint32)
    wl.batches += [W.Batch("insert", e, e), W.Batch("find", e), W.Batch("delete", e),
                   W.Batch("insert", ks, np.array([9, 10, 11, 12], dtype=np.uint32)),
                   W.Batch("find", np.array([EMPTY, 1, 5], dtype=np.uint32)),
                   W.Batch("insert", ks[1:], np.array([20, 21, 22], dtype=np.uint32)),
                   W.Batch("find", np.array([EMPTY], dtype=np.uint32)),
                   W.Batch("delete", np.array([EMPTY, 7, 2], dtype=np.uint32)),
                   W.Batch("insert", np.full(1, EMPTY, dtype=np.uint32), np.ones(1, dtype=np.uint32)),
                   W.Batch("find", np.array([2, 3, 0], dtype=np.uint32))]
    big = W.key_range(0, 2500, 5)
    wl.batches.append(W.Batch("insert", big, W.val_of(big, 1)))
    wl.batches.append(W.Batch("insert", big[::3], W.val_of(big[::3], 2)))   # mixed updates of a full-ish table
    wl.batches.append(W.Batch("find", np.concatenate([big, W.key_range(1 << 31, 900, 5)])))
    wl.batches.append(W.Batch("delete", big[:2400]))
    run_parity(oracle_mod, wl, B=8, binning=(1, 1, 1))


def test_binned_nullable_outputs_and_modes():
    """Nullable status / found / old-value outputs; mode 0 never bins; bad
    arguments are rejected."""
    from paper_conf_icde_lizlhs21_b200 import _lib as L
    import ctypes as C
    keys = W.key_range(0, 20000, 11)
    vals = W.val_of(keys, 0)
    g = Table(d=4, init_capacity=30000, alpha=0.3, beta=0.85, bucket_slots=8, binning=(1, 4, 8))
    kd, vd = dev(keys), dev(vals)
    L.check(L.dyc_insert_batch(g.handle, kd.data_ptr(), vd.data_ptr(), None, keys.size, None), "insert")
    out = torch.empty(keys.size, dtype=torch.int32, device="cuda")
    L.check(L.dyc_find_batch(g.handle, kd.data_ptr(), out.data_ptr(), None, keys.size, None), "find")
    np.testing.assert_array_equal(host_u32(out), vals)
    L.check(L.dyc_delete_batch(g.handle, kd[:5000].data_ptr(), None, None, 5000, None), "delete")
    assert g.stats()["m"] == keys.size - 5000
    assert g.binning_info()[0] == 3
    g.set_binning(0)
    v, f = g.find(kd)
    assert g.binning_info()[0] == 3
    np.testing.assert_array_equal(f.cpu().numpy(), (np.arange(keys.size) >= 5000).astype(np.uint8))
    with pytest.raises(L.DycError):
        g.set_binning(2)
    with pytest.raises(L.DycError):
        g.set_binning(0, 40, 0)
