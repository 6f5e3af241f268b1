"""Pins the CPU oracle (oracle/dyc_oracle.c) against things other than itself:
the brute-force map semantics of P:L188-189, the paper's invariants, and
scripted scenarios.  No GPU needed."""
import numpy as np
import pytest

from paper_conf_icde_lizlhs21_b200 import workload as W
from tests.bruteforce import BruteMap, EMPTY


def run_against_brute(oracle_mod, wl, B=4, policy=0, max_hops=64, check_every=True):
    o = oracle_mod.OracleTable(d=wl.d, init_capacity=wl.init_capacity, alpha=wl.alpha,
                               beta=wl.beta, bucket_slots=B, max_hops=max_hops, policy=policy)
    bm = BruteMap()
    fails = 0
    for i, b in enumerate(wl.batches):
        if b.op == "insert":
            np.testing.assert_array_equal(o.insert(b.keys, b.values), bm.insert(b.keys, b.values),
                                          err_msg=f"batch {i} insert status")
        elif b.op == "find":
            ov, of = o.find(b.keys)
            bv, bf = bm.find(b.keys)
            np.testing.assert_array_equal(of, bf, err_msg=f"batch {i} found")
            np.testing.assert_array_equal(ov, bv, err_msg=f"batch {i} values")
        else:
            ov, os_ = o.delete(b.keys)
            bv, bs = bm.delete(b.keys)
            np.testing.assert_array_equal(os_, bs, err_msg=f"batch {i} delete status")
            np.testing.assert_array_equal(ov, bv, err_msg=f"batch {i} old values")
        if check_every or i == len(wl.batches) - 1:
            np.testing.assert_array_equal(o.sorted_kv(), bm.sorted_kv(), err_msg=f"contents after {i}")
            bad, msg = o.check_invariants()
            assert bad == 0, f"batch {i}: {msg}"
            s = o.stats()
            # independent restatement of I5/I6 from the stats alone
            assert s["m"] == len(bm.m)
            assert max(s["buckets"]) <= 2 * min(s["buckets"]), "I6 (P:L312)"
            assert s["m"] <= wl.beta * s["N"], "I5 upper (P:L305)"
            assert s["max_probes"] <= 2, "I7 (P:L145)"
            failed_now, fails = s["n_fail_upsize"] != fails, s["n_fail_upsize"]
            if b.op != "find" and not failed_now and s["m"] < wl.alpha * s["N"]:
                # below alpha only if no subtable may be halved (Q13) or halving breaks beta
                t = max(range(wl.d), key=lambda j: (s["buckets"][j], j))
                n_t = s["buckets"][t]
                assert (n_t < 2 or n_t % 2 == 1
                        or s["m"] > wl.beta * (s["N"] - B * (n_t // 2))), "I5 lower (P:L305)"
    return o, bm


@pytest.mark.parametrize("seed", [1, 2, 3])
@pytest.mark.parametrize("d,B", [(2, 1), (3, 2), (4, 4), (4, 8), (8, 2), (5, 16)])
def test_random_streams_match_brute_force(oracle_mod, seed, d, B):
    alpha = round(min(0.3, 0.85 * d / (d + 1) - 0.01), 3)
    wl = W.random_op_stream(seed * 101 + d * 7 + B, n_batches=40, batch=300, universe=700,
                            d=d, alpha=alpha, beta=0.85, init_capacity=16)
    o, _ = run_against_brute(oracle_mod, wl, B=B)
    s = o.stats()
    assert s["n_upsize"] > 0 and s["n_downsize"] > 0


@pytest.mark.parametrize("seed", [11, 12])
def test_paper_weighted_policy_semantics(oracle_mod, seed):
    """The paper's randomized assignment changes placement only."""
    wl = W.random_op_stream(seed, n_batches=30, batch=400, universe=900, init_capacity=32)
    run_against_brute(oracle_mod, wl, B=4, policy=oracle_mod.oracle.PAPER_WEIGHTED)


def test_c1_config_matches_brute_force(oracle_mod):
    run_against_brute(oracle_mod, W.c1_rand_small())


def test_c2_shape_small_matches_brute_force(oracle_mod):
    wl = W.c2_rand_static(log2_n=15)
    o, _ = run_against_brute(oracle_mod, wl)
    s = o.stats()
    assert s["n_upsize"] == 0 and s["n_downsize"] == 0, "C2 is static (asserted no resize)"


def test_failure_path_never_drops_keys(oracle_mod):
    """L_max = 1 forces failed chains; the failure path must upsize and
    keep every key (Q17)."""
    wl = W.random_op_stream(77, n_batches=25, batch=500, universe=1000, init_capacity=8)
    o, _ = run_against_brute(oracle_mod, wl, B=1, max_hops=1)
    assert o.stats()["n_fail_upsize"] > 0


def test_reserved_key_and_empty_batches(oracle_mod):
    o = oracle_mod.OracleTable(init_capacity=64)
    bm = BruteMap()
    k = np.array([5, EMPTY, 7], dtype=np.uint32)
    v = np.array([50, 1, 70], dtype=np.uint32)
    np.testing.assert_array_equal(o.insert(k, v), bm.insert(k, v))
    assert o.insert(k, v).tolist() == [2, 0, 2]
    e = np.zeros(0, dtype=np.uint32)
    assert o.insert(e, e).size == 0
    ov, of = o.find(k)
    assert of.tolist() == [1, 0, 1] and ov.tolist() == [50, EMPTY, 70]
    dv, ds = o.delete(np.array([EMPTY, 5, 5], dtype=np.uint32))
    assert ds.tolist() == [0, 1, 0] and dv.tolist() == [EMPTY, 50, EMPTY]


def test_duplicate_keys_in_batch_sequential_last_wins(oracle_mod):
    """Reading Q9: oracle robustness semantics for a violated precondition."""
    o = oracle_mod.OracleTable(init_capacity=64)
    bm = BruteMap()
    k = np.array([9, 9, 10, 9], dtype=np.uint32)
    v = np.array([1, 2, 3, 4], dtype=np.uint32)
    np.testing.assert_array_equal(o.insert(k, v), bm.insert(k, v))
    np.testing.assert_array_equal(o.sorted_kv(), bm.sorted_kv())


def test_create_rejects_infeasible_bounds(oracle_mod):
    """Filled-factor analysis P:L315-318 (reading Q14: α ≤ βd/(d+1))."""
    with pytest.raises(ValueError):
        oracle_mod.OracleTable(d=4, alpha=0.69, beta=0.85)   # 0.85*4/5 = 0.68
    oracle_mod.OracleTable(d=4, alpha=0.67, beta=0.85).close()
    with pytest.raises(ValueError):
        oracle_mod.OracleTable(d=2, alpha=0.6, beta=0.85)    # 0.567
    with pytest.raises(ValueError):
        oracle_mod.OracleTable(d=1)


def test_cpp_brute_map_equals_python_dict():
    """The std::unordered_map baseline (oracle/brute_map.cpp)
    gives the dict model's results on a random stream with mixed batches."""
    import numpy as np
    from oracle import BruteMapCpp
    from paper_conf_icde_lizlhs21_b200 import workload as W
    from tests.bruteforce import BruteMap
    a, b = BruteMapCpp(), BruteMap()
    wl = W.random_op_stream(99, n_batches=30, batch=2000, universe=3000)
    for bt in wl.batches:
        if bt.op == "insert":
            np.testing.assert_array_equal(a.insert(bt.keys, bt.values), b.insert(bt.keys, bt.values))
        elif bt.op == "find":
            for x, y in zip(a.find(bt.keys), b.find(bt.keys)):
                np.testing.assert_array_equal(x, y)
        else:
            for x, y in zip(a.delete(bt.keys), b.delete(bt.keys)):
                np.testing.assert_array_equal(x, y)
    _, mixed = W.c4_zipf_mixed(U=20000, distinct=2000, grow_batches=3, cycles=1)
    for mb in mixed:
        for x, y in zip(a.mixed(mb.ops, mb.keys, mb.values), b.mixed(mb.ops, mb.keys, mb.values)):
            np.testing.assert_array_equal(x, y)
    assert len(a) == len(b.m)
