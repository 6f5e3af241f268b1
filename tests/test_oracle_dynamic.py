"""Oracle vs brute force on the dynamic configs' shapes (C3 sliding window,
C4 Zipf mixed batches, reading Q10 for mixed batches).  No GPU needed."""
import numpy as np

from paper_conf_icde_lizlhs21_b200 import workload as W
from tests.bruteforce import BruteMap
from tests.test_oracle_semantics import run_against_brute


def test_c3_shape_matches_brute_force(oracle_mod):
    wl = W.c3_dynamic(scale=0.0008, batch=4000, cycles=2, init_capacity=1024)
    o, _ = run_against_brute(oracle_mod, wl, B=8)
    s = o.stats()
    assert s["n_upsize"] > 0 and s["n_downsize"] > 0     # up- and downsizes repeat (C3)


def test_c4_mixed_matches_brute_force(oracle_mod):
    meta, batches = W.c4_zipf_mixed(U=40000, distinct=4000, grow_batches=5, cycles=2, init_capacity=1024)
    o = oracle_mod.OracleTable(d=4, init_capacity=meta.init_capacity, alpha=meta.alpha, beta=meta.beta,
                               bucket_slots=8)
    bm = BruteMap()
    for i, b in enumerate(batches):
        ov, os_ = o.mixed(b.ops, b.keys, b.values)
        bv, bs = bm.mixed(b.ops, b.keys, b.values)
        np.testing.assert_array_equal(os_, bs, err_msg=f"batch {i} status")
        np.testing.assert_array_equal(ov, bv, err_msg=f"batch {i} values")
        np.testing.assert_array_equal(o.sorted_kv(), bm.sorted_kv())
        assert o.check_invariants()[0] == 0
    assert o.stats()["n_downsize"] > 0


def test_mixed_phase_order(oracle_mod):
    """Reading Q10: a find sees the table before the batch, even when the same
    batch inserts other keys; statuses per op type."""
    o = oracle_mod.OracleTable(init_capacity=256)
    o.insert(np.array([1, 2], dtype=np.uint32), np.array([10, 20], dtype=np.uint32))
    ops = np.array([1, 0, 2, 0, 1], dtype=np.uint8)
    keys = np.array([3, 1, 2, 7, 1], dtype=np.uint32)
    vals = np.array([30, 0, 0, 0, 11], dtype=np.uint32)
    v, st = o.mixed(ops, keys, vals)
    assert st.tolist() == [1, 1, 1, 0, 2]
    assert v.tolist() == [0xFFFFFFFF, 10, 20, 0xFFFFFFFF, 0xFFFFFFFF]
    assert o.contents() == {1: 11, 3: 30}
