"""Brute-force map model of the KV-store semantics, written
independently of the oracle: a Python dict.  It pins the oracle's per-op
results and contents (SURVEY §8(c) "Semantic layer").

Semantics (readings Q7-Q10, Q25):
  insert(k,v): status 2 (UPDATED) if k present else 1 (INSERTED); M[k] = v.
               k == 0xFFFFFFFF (reserved EMPTY) -> status 0, no effect.
  find(k):     (M[k], 1) or (0xFFFFFFFF, 0)
  delete(k):   (old value, 1) and remove, or (0xFFFFFFFF, 0)
  Ops inside a batch apply in batch order (keys are distinct by precondition,
  which makes every order equivalent).
"""
import numpy as np

EMPTY = 0xFFFFFFFF


class BruteMap:
    def __init__(self):
        self.m = {}

    def insert(self, keys, vals):
        st = np.zeros(len(keys), dtype=np.uint8)
        for i, (k, v) in enumerate(zip(keys.tolist(), vals.tolist())):
            if k == EMPTY:
                continue
            st[i] = 2 if k in self.m else 1
            self.m[k] = v
        return st

    def find(self, keys):
        v = np.full(len(keys), EMPTY, dtype=np.uint32)
        f = np.zeros(len(keys), dtype=np.uint8)
        for i, k in enumerate(keys.tolist()):
            if k != EMPTY and k in self.m:
                v[i] = self.m[k]
                f[i] = 1
        return v, f

    def delete(self, keys):
        v = np.full(len(keys), EMPTY, dtype=np.uint32)
        st = np.zeros(len(keys), dtype=np.uint8)
        for i, k in enumerate(keys.tolist()):
            if k != EMPTY and k in self.m:
                v[i] = self.m.pop(k)
                st[i] = 1
        return v, st

    def mixed(self, ops, keys, vals):
        """Reading Q10: finds see the pre-batch map, then inserts, then deletes."""
        v = np.full(len(keys), EMPTY, dtype=np.uint32)
        st = np.zeros(len(keys), dtype=np.uint8)
        for op in (0, 1, 2):
            sel = np.nonzero(ops == op)[0]
            if op == 0:
                v[sel], st[sel] = self.find(keys[sel])
            elif op == 1:
                st[sel] = self.insert(keys[sel], vals[sel])
            else:
                v[sel], st[sel] = self.delete(keys[sel])
        return v, st

    def sorted_kv(self):
        ks = np.array(sorted(self.m), dtype=np.uint64)
        vs = np.array([self.m[int(k)] for k in ks], dtype=np.uint64)
        return ks | (vs << np.uint64(32))


def replay_sizes(d, B, init_capacity, alpha, beta, m_after_batches):
    """Closed-form replay of the resize policy from the live-key count alone
    (double the smallest / halve the largest while theta leaves
    [alpha, beta]; readings Q11-Q13).  `m_after_batches` lists, per batch,
    (kind, m_before_placement_target, m_after) where for inserts the target is
    m + n_new.  Returns the per-batch subtable sizes.  Valid while no
    failure-triggered upsize happens (checked by the caller)."""
    per = max(1, -(-init_capacity // (d * B)))
    n = [per] * d
    out = []
    for kind, target, m in m_after_batches:
        if kind == "empty":          # reading Q32: an empty batch is a no-op
            out.append(list(n))
            continue
        if kind == "insert":
            while target > beta * (B * sum(n)):
                t = min(range(d), key=lambda i: (n[i], i))
                n[t] *= 2
        while m < alpha * (B * sum(n)):
            t = max(range(d), key=lambda i: (n[i], i))
            if n[t] < 2 or n[t] % 2:
                break
            if m > beta * (B * (sum(n) - n[t] // 2)):
                break
            n[t] //= 2
        out.append(list(n))
    return out
