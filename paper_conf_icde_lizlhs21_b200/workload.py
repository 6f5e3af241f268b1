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


def perm_pow2(x: np.ndarray, log2n: int, seed: int) -> np.ndarray:
    """A seeded bijection on [0, 2^log2n): xor-shift and odd-multiply rounds
    (each invertible mod 2^log2n).  Used instead of shuffles so that 2^27-op
    batches are generated in O(n) vectorised passes."""
    mask = np.uint64((1 << log2n) - 1)
    sh = np.uint64(max(1, (log2n + 1) // 2))
    x = (np.asarray(x, dtype=np.uint64) ^ np.uint64(seed & ((1 << log2n) - 1))) & mask
    with np.errstate(over="ignore"):
        for c in (0x2C1B3C6D, 0x297A2D39, 0x9E3779B1):
            x ^= x >> sh
            x = (x * np.uint64(c)) & mask
        x ^= x >> sh
    return x


def c2_rand_static(log2_n: int = 27, seed_cfg: Optional[int] = None,
                   beta: float = 0.85) -> Workload:
    """Config C2 (BASELINE.json configs[1]): 2^27 inserts into a table sized for
    fill beta, then 2^27 finds (50% hit: 2^26 distinct live keys and 2^26 misses,
    interleaved pseudo-randomly) and 2^26 deletes of distinct live keys.
    `log2_n` scales it down for parity tests."""
    s = config_seed(2) if seed_cfg is None else seed_cfg
    n = 1 << log2_n
    keys = key_range(0, n, s)
    vals = val_of(keys, 0)
    cap = int(math.ceil(n / beta))
    w = Workload(f"C2-rand-static-2^{log2_n}", 4, 0.3, beta, cap)
    w.batches.append(Batch("insert", keys, vals))
    i = np.arange(n, dtype=np.uint64)
    j = perm_pow2(i, log2_n, s ^ 0x1234567)            # position -> draw index
    half = np.uint64(n // 2)
    hit = j < half
    hit_idx = perm_pow2(j, log2_n, s ^ 0x7654321)      # distinct indices of live keys
    q = np.where(hit, keys[hit_idx.astype(np.int64) & (n - 1)],
                 key_of(np.uint64(MISS_BASE) + (j - half), s)).astype(np.uint32)
    # the miss range may contain the single EMPTY preimage: replace it by a live key's twin miss
    q[q == np.uint32(EMPTY_KEY)] = key_of(np.array([MISS_BASE + n], dtype=np.uint64), s)[0]
    w.batches.append(Batch("find", q))
    del_idx = perm_pow2(np.arange(n // 2, dtype=np.uint64), log2_n, s ^ 0x5A5A5A5)
    w.batches.append(Batch("delete", np.ascontiguousarray(keys[del_idx.astype(np.int64)])))
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


# ---------------------------------------------------------------------------
# The same C2 recipe evaluated with torch int64 tensor ops (on the GPU or on
# many CPU threads), for the full 2^27-op benchmark batches.  Bit-identical to
# c2_rand_static (tests/test_workload.py); still no arithmetic of the method.
def _lowbias32_t(x):
    m = 0xFFFFFFFF
    x = x ^ (x >> 16)
    x = (x * 0x7FEB352D) & m
    x = x ^ (x >> 15)
    x = (x * 0x846CA68B) & m
    x = x ^ (x >> 16)
    return x


def _key_of_t(idx, seed):
    return _lowbias32_t((idx & 0xFFFFFFFF) ^ (seed & 0xFFFFFFFF))


def _perm_pow2_t(x, log2n, seed):
    mask = (1 << log2n) - 1
    sh = max(1, (log2n + 1) // 2)
    x = (x ^ (seed & mask)) & mask
    for c in (0x2C1B3C6D, 0x297A2D39, 0x9E3779B1):
        x = x ^ (x >> sh)
        x = (x * c) & mask
    return x ^ (x >> sh)


def _as_i32(x):
    import torch
    return torch.where(x >= (1 << 31), x - (1 << 32), x).to(torch.int32)


def c2_rand_static_torch(log2_n: int = 27, device="cuda", seed_cfg: Optional[int] = None, beta: float = 0.85,
                         key_base: int = 0, miss_base: int = 0):
    """Returns (init_capacity, ins_keys, ins_vals, find_keys, del_keys) as int32
    tensors holding the uint32 bit patterns of c2_rand_static(log2_n).
    key_base / miss_base shift the key index ranges (disjoint per-rank batches
    for the sharded bench: key(key_base + i), misses key(2^31 + miss_base + j))."""
    import torch
    s = config_seed(2) if seed_cfg is None else seed_cfg
    n = 1 << log2_n
    idx = key_base + torch.arange(n + 1, dtype=torch.int64, device=device)
    k = _key_of_t(idx, s)
    k = k[k != EMPTY_KEY][:n]                                    # key_range(0, n, s)
    mix = (0x9E3779B9 * 1) & 0xFFFFFFFF
    v = _lowbias32_t(k ^ mix)                                    # val_of(keys, 0)
    i = torch.arange(n, dtype=torch.int64, device=device)
    j = _perm_pow2_t(i, log2_n, s ^ 0x1234567)
    hit = j < n // 2
    hit_idx = _perm_pow2_t(j, log2_n, s ^ 0x7654321) & (n - 1)
    miss = _key_of_t(MISS_BASE + miss_base + (j - n // 2), s)
    q = torch.where(hit, k[hit_idx], miss)
    q = torch.where(q == EMPTY_KEY, _key_of_t(torch.tensor(MISS_BASE + miss_base + n, device=device), s), q)
    del_idx = _perm_pow2_t(torch.arange(n // 2, dtype=torch.int64, device=device), log2_n, s ^ 0x5A5A5A5)
    dk = k[del_idx]
    cap = int(math.ceil(n / beta))
    return cap, _as_i32(k), _as_i32(v), _as_i32(q), _as_i32(dk)


def wide_static_torch(log2_n: int = 26, value_words: int = 2, device="cuda", beta: float = 0.85):
    """C2's shape for the wide-key table (NEXT-3): 64-bit keys whose low half is
    C2's key (distinct, so the 64-bit keys are distinct and misses stay misses)
    and whose high half is a second mix of it; values of W words.  Returns
    (init_capacity, keys i64[n], values i64[n, W], find_keys i64[n] (50% hit),
    del_keys i64[n/2])."""
    import torch
    cap, k, _, q, dk = c2_rand_static_torch(log2_n, device=device, beta=beta)

    def widen(x32):
        lo = x32.to(torch.int64) & 0xFFFFFFFF
        hi = _lowbias32_t(lo ^ 0x6A09E667)
        return (hi << 32) | lo                       # int64 bit pattern of the u64 key

    kw = widen(k)
    vals = torch.stack([kw * (2 * w + 3) + w for w in range(value_words)], dim=1).contiguous()
    return cap, kw, vals, widen(q), widen(dk)


# ---------------------------------------------------------------------------
# Config C3: TW/RE-shaped dynamic stream (§VI-A "Dynamic Hashing
# Comparison"; datasets Table `table:exp_data_sets` P:L671-672).
def c3_dynamic(scale: float = 1.0, shape: str = "TW", batch: int = 1_000_000, r: float = 0.2,
               cycles: int = 2, seed_cfg: Optional[int] = None, init_capacity: int = 1 << 20) -> Workload:
    """Insert stream shaped like TW (50,876,784 ops over 44,523,684 unique keys,
    multiplicity <= 4) or RE (48,104,875 / 41,466,682, <= 2), scaled by `scale`.
    Each step: one insert batch (distinct keys), one find batch of `batch` ops
    (50% live / 50% never inserted), one delete batch of r*batch OLDEST live keys
    (sliding window; r = #delete/#insert, reading Q22).  After the
    stream is exhausted the batches are replayed with insert and delete key sets
    swapped (reading Q27); `cycles` repeats forward stream + swap pass.
    Vectorised (numpy) so the full-size stream is generated in seconds."""
    s = config_seed(3) if seed_cfg is None else seed_cfg
    rng = np.random.Generator(np.random.PCG64(s))
    total, uniq, mult = {"TW": (50_876_784, 44_523_684, 4), "RE": (48_104_875, 41_466_682, 2)}[shape]
    T, U = max(1, int(total * scale)), max(1, int(uniq * scale))
    batch = max(1, int(batch))
    keys = key_range(0, U, s)
    n_batches = (U + batch - 1) // batch
    # repeats: T-U extra occurrences, each key at most mult-1 times, each in a
    # strictly later batch than the key's previous occurrence
    rep = rng.choice(U, size=min(T - U, U * (mult - 1)), replace=True)
    cnt = np.minimum(np.bincount(rep, minlength=U), mult - 1)
    rep_ids, rep_batch = [], []
    cur = np.arange(U) // batch
    for j in range(mult - 1):
        sel = np.nonzero(cnt > j)[0]
        cur_sel = cur[sel] + 1 + rng.integers(0, 3, size=sel.size)
        cur[sel] = cur_sel
        rep_ids.append(sel)
        rep_batch.append(cur_sel)
    rep_ids = np.concatenate(rep_ids) if rep_ids else np.zeros(0, np.int64)
    rep_batch = np.concatenate(rep_batch) if rep_batch else np.zeros(0, np.int64)
    nb_total = int(max(n_batches, rep_batch.max() + 1 if rep_batch.size else 0))
    order_rb = np.argsort(rep_batch, kind="stable")
    rep_ids, rep_batch = rep_ids[order_rb], rep_batch[order_rb]
    rep_bounds = np.searchsorted(rep_batch, np.arange(nb_total + 1))
    w = Workload(f"C3-{shape}-x{scale:g}", 4, 0.3, 0.85, init_capacity)
    # FIFO of live keys by insertion time: order[] holds key ids, live_pos[kid]
    # the position of the key's current life (-1 when not live)
    order = np.empty(T + 1, dtype=np.int64)
    tail = head = 0
    live_pos = np.full(U, -1, dtype=np.int64)
    nlive = 0
    ins_batches, del_batches = [], []
    miss_ctr = 0
    for b in range(nb_total):
        fresh = np.arange(b * batch, min((b + 1) * batch, U)) if b < n_batches else np.zeros(0, np.int64)
        ids_b = np.unique(np.concatenate([fresh, rep_ids[rep_bounds[b]:rep_bounds[b + 1]]]))
        if ids_b.size == 0:
            continue
        ins_batches.append(ids_b)
        w.batches.append(Batch("insert", keys[ids_b], val_of(keys[ids_b], b + 1)))
        new = ids_b[live_pos[ids_b] < 0]                   # first life or re-insert after delete
        order[tail:tail + new.size] = new
        live_pos[new] = np.arange(tail, tail + new.size)
        tail += new.size
        nlive += new.size
        # finds: half live (sampled), half never inserted
        nh = min(batch // 2, nlive)
        hits = np.zeros(0, np.int64)
        while hits.size < nh:
            cand_pos = rng.integers(head, tail, size=2 * (nh - hits.size) + 16)
            cand = order[cand_pos]
            ok = live_pos[cand] == cand_pos
            hits = np.unique(np.concatenate([hits, cand[ok]]))[:nh] if hits.size else np.unique(cand[ok])[:nh]
        miss = key_range(MISS_BASE + miss_ctr, batch - hits.size, s)
        miss_ctr += batch - hits.size
        q = np.concatenate([keys[hits], miss])
        rng.shuffle(q)
        w.batches.append(Batch("find", q))
        # deletes: the r*batch oldest live keys
        nd = min(int(r * batch), nlive)
        got = []
        need = nd
        while need > 0:
            seg = order[head:min(tail, head + 2 * need + 64)]
            pos = np.arange(head, head + seg.size)
            ok = live_pos[seg] == pos
            take = np.nonzero(ok)[0][:need]
            if take.size:
                got.append(seg[take])
                head = pos[take[-1]] + 1
                need -= take.size
            else:
                head += seg.size
        dl = np.concatenate(got) if got else np.zeros(0, np.int64)
        live_pos[dl] = -1
        nlive -= dl.size
        del_batches.append(dl)
        w.batches.append(Batch("delete", keys[dl]))
    base = list(w.batches)
    for c in range(cycles):
        if c > 0:
            for bt in base:       # replay the forward stream
                w.batches.append(Batch(bt.op, bt.keys.copy(), None if bt.values is None else bt.values.copy()))
        for b, ids_b in enumerate(ins_batches):                # swap pass
            d_ids = del_batches[b]
            w.batches.append(Batch("insert", keys[d_ids], val_of(keys[d_ids], 1000 * (c + 1) + b)))
            w.batches.append(Batch("delete", keys[ids_b]))
    return w


# ---------------------------------------------------------------------------
# Config C4: LINE/COM-shaped Zipf(0.99) mixed batches.
@dataclass
class MixedBatch:
    ops: np.ndarray      # uint8: 0 find, 1 insert, 2 delete
    keys: np.ndarray     # uint32, distinct within the batch
    values: np.ndarray   # uint32


def zipf_distinct(rng, cdf: np.ndarray, count: int, exclude: Optional[np.ndarray] = None) -> np.ndarray:
    """Draw Zipf ranks (inverse CDF) until `count` distinct ranks are collected,
    in first-draw order (vectorised with a seen-mask over the universe)."""
    seen = np.zeros(cdf.size + 1, dtype=bool)
    if exclude is not None and len(exclude):
        seen[np.asarray(exclude, dtype=np.int64)] = True
    got = []
    have = 0
    while have < count:
        draw = np.searchsorted(cdf, rng.random(max(4096, 2 * (count - have))), side="right")
        draw = draw[~seen[draw]]
        if draw.size == 0:
            continue
        _, first = np.unique(draw, return_index=True)
        new = draw[np.sort(first)][:count - have]
        seen[new] = True
        got.append(new)
        have += new.size
    return np.concatenate(got).astype(np.int64)


def c4_zipf_mixed(U: int = 45_159_880, distinct: int = 4_000_000, grow_batches: int = 16, cycles: int = 2,
                  exponent: float = 0.99, seed_cfg: Optional[int] = None, init_capacity: int = 1 << 20,
                  drain_floor: float = 0.10, max_drain: int = 64):
    """Mixed 50/30/20 find/insert/delete batches over Zipf(0.99) ranks of a
    universe of U keys (LINE-shaped: U = 45,159,880; COM-shaped: U = 4,583,941
    with 1M-distinct batches).  Grow phase: `grow_batches` batches; drain phase:
    50% find / 5% insert / 45% delete (deletes drawn from the live set) until
    the live count is below drain_floor of its peak.  Returns (Workload meta, list of
    MixedBatch)."""
    s = config_seed(4) if seed_cfg is None else seed_cfg
    rng = np.random.Generator(np.random.PCG64(s))
    ranks = np.arange(1, U + 1, dtype=np.float64)
    cdf = np.cumsum(ranks ** (-exponent))
    cdf /= cdf[-1]
    keys_of = lambda r: key_of(np.asarray(r, dtype=np.uint64), s)  # noqa: E731  (rank -> key, a bijection)
    meta = Workload(f"C4-zipf-U{U}", 4, 0.3, 0.85, init_capacity)
    out = []
    live = np.zeros(U + 1, dtype=bool)
    nlive = 0
    ver = 0

    def apply(r, ops):
        nonlocal nlive
        ins, dl = r[ops == 1], r[ops == 2]
        nlive += int((~live[ins]).sum()) - int(live[dl].sum())
        live[ins] = True
        live[dl] = False

    for c in range(cycles):
        for b in range(grow_batches):
            ver += 1
            r = zipf_distinct(rng, cdf, distinct)
            u = rng.random(r.size)
            ops = np.where(u < 0.5, 0, np.where(u < 0.8, 1, 2)).astype(np.uint8)
            k = keys_of(r)
            out.append(MixedBatch(ops, k, val_of(k, ver)))
            apply(r, ops)
        peak = nlive
        for _ in range(max_drain):
            if nlive <= drain_floor * peak or nlive == 0:
                break
            ver += 1
            nd = min(nlive, int(0.45 * distinct))
            lv = np.nonzero(live)[0]
            dl = rng.choice(lv, size=nd, replace=False)
            rest = zipf_distinct(rng, cdf, distinct - nd, exclude=dl)
            u = rng.random(rest.size)
            ops_rest = np.where(u < 0.5 / 0.55, 0, 1).astype(np.uint8)      # 50 find : 5 insert
            r = np.concatenate([dl, rest])
            ops = np.concatenate([np.full(nd, 2, np.uint8), ops_rest])
            perm = rng.permutation(r.size)
            r, ops = r[perm], ops[perm]
            k = keys_of(r)
            out.append(MixedBatch(ops, k, val_of(k, ver)))
            apply(r, ops)
    return meta, out


# ---------------------------------------------------------------------------
# Config C5: RAND 2^31 keys hash-partitioned across G GPUs.
def c5_batches_torch(rank: int, world: int, device="cuda", log2_keys: int = 31, batch: int = 1 << 24,
                     fill_batches: Optional[int] = None, mixed_batches: int = 32, seed_cfg: Optional[int] = None):
    """Generator of this rank's slice of every global batch (rank r issues ops
    [r*batch/G, (r+1)*batch/G) of each).  Fill: key(0 .. 2^log2_keys - 1) in
    global batches of `batch` inserts.  Then mixed 50/30/20 global batches:
    finds = half live keys key(2^(log2_keys-1) + perm(j)) (a range no mixed batch
    deletes) and half never-inserted misses; inserts = new keys from the index
    range above the fill; deletes = distinct live keys key(b*0.2*batch + j).
    Keys are distinct within every global batch.  Yields (op, keys, values)
    int32 tensors; op in {"insert", "mixed"}; a mixed batch is (ops u8, keys, vals)."""
    import torch
    s = config_seed(5) if seed_cfg is None else seed_cfg
    n_keys = 1 << log2_keys
    fb = fill_batches if fill_batches is not None else n_keys // batch
    lo, hi = rank * batch // world, (rank + 1) * batch // world
    loc = torch.arange(lo, hi, dtype=torch.int64, device=device)
    for j in range(fb):
        k = _key_of_t(j * batch + loc, s)
        yield "insert", _as_i32(k), _as_i32(_lowbias32_t(k ^ 0x9E3779B9))
    nf, ni = batch // 2, (batch * 3) // 10
    nd = batch - nf - ni
    half = n_keys >> 1
    for b in range(mixed_batches):
        g = loc                                               # this rank's positions in the global batch
        is_f, is_i = g < nf, (g >= nf) & (g < nf + ni)
        # finds: even positions live (from [half, n_keys)), odd positions misses
        live_idx = half + (_perm_pow2_t(g, log2_keys - 1, s ^ (b * 7919 + 1)) & (half - 1))
        miss_idx = n_keys + (1 << 30) + b * batch + g
        f_idx = torch.where(g % 2 == 0, live_idx, miss_idx)
        i_idx = n_keys + b * ni + (g - nf)                    # new keys above the fill range
        d_idx = b * nd + (g - nf - ni)                        # distinct live keys below `half`
        idx = torch.where(is_f, f_idx, torch.where(is_i, i_idx, d_idx))
        k = _key_of_t(idx, s)
        ops = torch.where(is_f, 0, torch.where(is_i, 1, 2)).to(torch.uint8)
        yield "mixed", ops, _as_i32(k), _as_i32(_lowbias32_t(k ^ (0x9E3779B9 * (b + 2) & 0xFFFFFFFF)))
