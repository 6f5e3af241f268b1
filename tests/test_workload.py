"""The torch evaluation of the C2 generator equals the numpy one (CPU)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from paper_conf_icde_lizlhs21_b200 import workload as W


@pytest.mark.parametrize("log2_n", [10, 16])
def test_c2_torch_matches_numpy(log2_n):
    wl = W.c2_rand_static(log2_n)
    cap, k, v, q, dk = W.c2_rand_static_torch(log2_n, device="cpu")
    assert cap == wl.init_capacity
    ins, fnd, dele = wl.batches
    np.testing.assert_array_equal(k.numpy().view(np.uint32), ins.keys)
    np.testing.assert_array_equal(v.numpy().view(np.uint32), ins.values)
    np.testing.assert_array_equal(q.numpy().view(np.uint32), fnd.keys)
    np.testing.assert_array_equal(dk.numpy().view(np.uint32), dele.keys)


def test_c2_shape():
    wl = W.c2_rand_static(14)
    ins, fnd, dele = wl.batches
    n = ins.keys.size
    assert len(np.unique(ins.keys)) == n and (ins.keys != W.EMPTY_KEY).all()
    assert np.isin(fnd.keys, ins.keys).sum() == n // 2          # 50% hit (Q23)
    assert len(np.unique(fnd.keys)) == n
    assert len(np.unique(dele.keys)) == n // 2 and np.isin(dele.keys, ins.keys).all()


def test_c1_shape():
    wl = W.c1_rand_small()
    ops = [b.op for b in wl.batches]
    assert ops == ["insert"] * 8 + ["find"] * 8 + ["delete"] * 8
    allk = np.concatenate([b.keys for b in wl.batches if b.op == "insert"])
    assert len(np.unique(allk)) == 65536
    for b in wl.batches:
        assert len(np.unique(b.keys)) == b.keys.size == 8192
