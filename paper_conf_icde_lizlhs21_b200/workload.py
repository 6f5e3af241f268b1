"""Seeded synthetic workload generators (shared by the CUDA path, the oracle and the tests).

This module holds NO arithmetic of the method (no table hashing, no placement,
no resize policy): it only produces keys, values and op streams shaped like the
paper's workloads, so that both sides of every parity test consume the same
input.  Recipes follow SURVEY.md §8(d) and are restated in DESIGN.md §3.

Paper workloads (§VI-A, Table `table:exp_data_sets` L654-677,
parameters Table `tbl:parameters` L739-753):

* RAND: 100M distinct keys (L675, L687).  Reading Q24: uniform distinct u32 keys
  through a seeded bijection (a narrow normal cannot give 2^31 distinct keys).
* static: insert everything, then random finds (L700-702); reading Q23: 50% hit.
* dynamic: batches of 1M inserts + 1M finds + r*1M deletes (L729-737).
* LINE/COM: Zipf-shaped key multiplicities (L673-674); here Zipf(0.99).

Generator primitives:
    lowbias32(x)    : x^=x>>16; x*=0x7feb352d; x^=x>>15; x*=0x846ca68b; x^=x>>16
    key(i; s)       : lowbias32(i ^ s), a bijection on u32; the one index whose
                      key is 0xFFFFFFFF (the reserved EMPTY key) is skipped
    val(k, ver)     : lowbias32(k ^ (0x9E3779B9*(ver+1) mod 2^32))
    seed s_c        : 0xD7C00000 + config number
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field
from typing import List, Optional

import numpy as np

EMPTY_KEY = 0xFFFFFFFF
MISS_BASE = 1 << 31          # miss keys are key(2^31 + j): disjoint from inserted indices < 2^31
_U32 = np.uint32


def config_seed(config_no: int) -> int:
    return (0xD7C00000 + int(config_no)) & 0xFFFFFFFF


def lowbias32(x: np.ndarray) -> np.ndarray:
    """Chris Wellons' lowbias32 integer permutation, vectorised on uint32."""
    x = np.asarray(x, dtype=_U32).copy()
    with np.errstate(over="ignore"):
        x ^= x >> _U32(16)
        x *= _U32(0x7FEB352D)
        x ^= x >> _U32(15)
        x *= _U32(0x846CA68B)
        x ^= x >> _U32(16)
    return x


def key_of(idx: np.ndarray, seed: int) -> np.ndarray:
    """key(i; s) = lowbias32(i ^ s); may return EMPTY for exactly one i."""
    return lowbias32(np.asarray(idx, dtype=np.uint64).astype(_U32) ^ _U32(seed))


def key_range(start: int, count: int, seed: int) -> np.ndarray:
    """Distinct keys key(start..), skipping the single index that maps to EMPTY."""
    idx = np.arange(start, start + count + 1, dtype=np.uint64)
    k = key_of(idx, seed)
    k = k[k != _U32(EMPTY_KEY)]
    return np.ascontiguousarray(k[:count])


def val_of(keys: np.ndarray, ver: int) -> np.ndarray:
    mix = _U32((0x9E3779B9 * (ver + 1)) & 0xFFFFFFFF)
    return lowbias32(np.asarray(keys, dtype=_U32) ^ mix)


@dataclass
class Batch:
    op: str                      # "insert" | "find" | "delete"
    keys: np.ndarray             # uint32[n]
    values: Optional[np.ndarray] = None   # uint32[n] for inserts


@dataclass
class Workload:
    name: str
    d: int
    alpha: float
    beta: float
    init_capacity: int
    batches: List[Batch] = field(default_factory=list)
    note: str = ""

    @property
    def n_ops(self) -> int:
        return sum(int(b.keys.size) for b in self.batches)


def c1_rand_small(seed_cfg: Optional[int] = None, n_keys: int = 65536,
                  batch: int = 8192) -> Workload:
    """Config C1 (BASELINE.json configs[0]): 65,536 keys, d=4, alpha=0.5, beta=0.85,
    8 insert batches of 8,192, 8 find batches (50% hit), 8 delete batches."""
    s = config_seed(1) if seed_cfg is None else seed_cfg
    rng = np.random.Generator(np.random.PCG64(s))
    keys = key_range(0, n_keys, s)
    vals = val_of(keys, 0)
    w = Workload("C1-rand-small", 4, 0.5, 0.85, 4096)
    nb = n_keys // batch
    for i in range(nb):
        sl = slice(i * batch, (i + 1) * batch)
        w.batches.append(Batch("insert", keys[sl].copy(), vals[sl].copy()))
    half = batch // 2
    for i in range(nb):
        hits = keys[rng.choice(n_keys, size=half, replace=False)]
        miss = key_range(MISS_BASE + i * half, half, s)
        q = np.concatenate([hits, miss])
        rng.shuffle(q)
        w.batches.append(Batch("find", q))
    order = rng.permutation(n_keys)
    for i in range(nb):
        w.batches.append(Batch("delete", keys[order[i * batch:(i + 1) * batch]].copy()))
    return w


def c2_rand_static(log2_n: int = 27, seed_cfg: Optional[int] = None,
                   beta: float = 0.85) -> Workload:
    """Config C2 (BASELINE.json configs[1]): 2^27 inserts into a table sized for
    fill beta, then 2^27 finds (50% hit, shuffled) and 2^26 deletes of live keys.
    `log2_n` scales it down for parity tests."""
    s = config_seed(2) if seed_cfg is None else seed_cfg
    n = 1 << log2_n
    rng = np.random.Generator(np.random.PCG64(s))
    keys = key_range(0, n, s)
    vals = val_of(keys, 0)
    cap = int(math.ceil(n / beta))
    w = Workload(f"C2-rand-static-2^{log2_n}", 4, 0.3, beta, cap)
    w.batches.append(Batch("insert", keys, vals))
    perm = rng.permutation(n)
    hits = keys[perm[: n // 2]]
    miss = key_range(MISS_BASE, n // 2, s)
    q = np.concatenate([hits, miss])
    rng.shuffle(q)
    w.batches.append(Batch("find", q))
    w.batches.append(Batch("delete", keys[perm[n // 2: n // 2 + n // 2]].copy()))
    return w


def random_op_stream(seed: int, n_batches: int, batch: int, universe: int,
                     d: int = 4, alpha: float = 0.3, beta: float = 0.85,
                     init_capacity: int = 64, drain: bool = True) -> Workload:
    """Random single-type batches over a small key universe (keys distinct within
    a batch; updates, re-inserts and misses all occur).  Used by parity tests."""
    rng = np.random.Generator(np.random.PCG64(seed))
    univ = key_range(0, universe, seed & 0xFFFFFFFF)
    w = Workload(f"random-{seed}", d, alpha, beta, init_capacity)
    for i in range(n_batches):
        op = ("insert", "insert", "find", "delete")[int(rng.integers(0, 4))]
        n = int(rng.integers(0, batch + 1))
        k = univ[rng.choice(universe, size=min(n, universe), replace=False)]
        if op == "insert":
            w.batches.append(Batch(op, k, val_of(k, i + 1)))
        else:
            w.batches.append(Batch(op, k))
    if drain:   # delete the whole universe so the shrinking path (downsizes) runs
        order = rng.permutation(universe)
        for j in range(0, universe, max(1, batch)):
            w.batches.append(Batch("delete", univ[order[j:j + batch]].copy()))
    return w
