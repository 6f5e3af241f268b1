"""world_size-2 gloo test of the sharded router's orchestration (DistTable):
count exchange, splits, forward and reverse all-to-all, unpermute.  The per-rank
table is an injected CPU stand-in (a dict with key % world routing); the CUDA
routing kernels are covered by tests/test_gpu_dist.py.  No GPU needed."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

EMPTY = 0xFFFFFFFF


class DictShard:
    """CPU stand-in with the Table routing/batch interface (test double)."""

    def __init__(self):
        self.m = {}

    def route_count(self, keys, world):
        k = keys.to(torch.int64) & 0xFFFFFFFF
        return torch.bincount(k % world, minlength=world).to(torch.int64)

    def route_scatter(self, keys, values, world, counts, tags=None):
        k = keys.to(torch.int64) & 0xFFFFFFFF
        dest = k % world
        order = torch.argsort(dest, stable=True)
        pos = torch.empty_like(order)
        pos[order] = torch.arange(order.numel())
        kout = keys[order].clone()
        vout = values[order].clone() if values is not None else None
        if tags is not None:
            return kout, vout, pos.to(torch.int32), tags[order].clone()
        return kout, vout, pos.to(torch.int32)

    def mixed(self, ops, keys, vals):
        v = torch.full((keys.numel(),), -1, dtype=torch.int32)
        s = torch.zeros(keys.numel(), dtype=torch.uint8)
        for op in (0, 1, 2):
            sel = torch.nonzero(ops == op).flatten()
            if sel.numel() == 0:
                continue
            if op == 0:
                v[sel], s[sel] = self.find(keys[sel])
            elif op == 1:
                s[sel] = self.insert(keys[sel], vals[sel])
            else:
                v[sel], s[sel] = self.delete(keys[sel])
        return v, s

    def route_unpermute(self, pos, rv=None, rs=None, out_vals=None, out_status=None):
        p = pos.to(torch.int64)
        v = rv[p] if rv is not None else None
        s = rs[p] if rs is not None else None
        if out_vals is not None and v is not None:
            out_vals.copy_(v)
            v = out_vals
        if out_status is not None and s is not None:
            out_status.copy_(s)
            s = out_status
        return v, s

    def insert(self, keys, vals):
        st = torch.zeros(keys.numel(), dtype=torch.uint8)
        for i, (k, v) in enumerate(zip(keys.tolist(), vals.tolist())):
            k &= 0xFFFFFFFF
            if k == EMPTY:
                continue
            st[i] = 2 if k in self.m else 1
            self.m[k] = v
        return st

    # one batch in parts: the stand-in applies each part immediately
    def insert_begin(self, n):
        pass

    def insert_part(self, keys, vals):
        return self.insert(keys, vals)

    def insert_end(self):
        pass

    def delete_begin(self, n):
        pass

    def delete_part(self, keys):
        return self.delete(keys)

    def delete_end(self):
        pass

    def find(self, keys):
        v = torch.full((keys.numel(),), -1, dtype=torch.int32)
        f = torch.zeros(keys.numel(), dtype=torch.uint8)
        for i, k in enumerate(keys.tolist()):
            k &= 0xFFFFFFFF
            if k in self.m:
                v[i], f[i] = self.m[k], 1
        return v, f

    def delete(self, keys):
        v = torch.full((keys.numel(),), -1, dtype=torch.int32)
        s = torch.zeros(keys.numel(), dtype=torch.uint8)
        for i, k in enumerate(keys.tolist()):
            k &= 0xFFFFFFFF
            if k in self.m:
                v[i], s[i] = self.m.pop(k), 1
        return v, s


def _batches(world, nb=6, per=200, seed=3):
    """Deterministic per-rank batches; keys distinct across ranks within a batch."""
    rng = np.random.Generator(np.random.PCG64(seed))
    univ = rng.choice(1 << 31, size=3000, replace=False).astype(np.int64)
    out = []
    for b in range(nb):
        op = ["insert", "find", "insert", "delete", "find", "delete"][b % 6]
        ks = rng.choice(univ, size=per * world, replace=False)
        vs = rng.integers(0, 1 << 31, size=per * world)
        out.append((op, [ks[r * per:(r + 1) * per] for r in range(world)],
                    [vs[r * per:(r + 1) * per] for r in range(world)]))
    return out


def _worker(rank, world, port, q, chunks):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icde_lizlhs21_b200.dist import DistTable
    dt = DistTable(DictShard(), chunks=chunks)
    model = {}
    ok = True
    for op, ks, vs in _batches(world):
        mine = torch.tensor(ks[rank], dtype=torch.int32)
        if op == "insert":
            st = dt.insert(mine, torch.tensor(vs[rank], dtype=torch.int32))
            exp = [2 if int(k) in model else 1 for k in ks[rank]]
            ok &= st.tolist() == exp
            for r in range(world):
                for k, v in zip(ks[r], vs[r]):
                    model[int(k)] = int(v)
        elif op == "find":
            v, f = dt.find(mine)
            ok &= f.tolist() == [1 if int(k) in model else 0 for k in ks[rank]]
            ok &= [int(x) for x, h in zip(v.tolist(), f.tolist()) if h] == [model[int(k)] for k in ks[rank] if int(k) in model]
        else:
            v, s = dt.delete(mine)
            ok &= s.tolist() == [1 if int(k) in model else 0 for k in ks[rank]]
            for r in range(world):
                for k in ks[r]:
                    model.pop(int(k), None)
    # one mixed batch (find -> insert -> delete, reading Q10), keys distinct across ranks
    rng = np.random.Generator(np.random.PCG64(99))
    allk = rng.choice(np.arange(1, 1 << 20), size=300 * world, replace=False)
    allops = rng.integers(0, 3, size=allk.size)
    mk = torch.tensor(allk[rank * 300:(rank + 1) * 300], dtype=torch.int32)
    mo = torch.tensor(allops[rank * 300:(rank + 1) * 300], dtype=torch.uint8)
    mv = torch.arange(300, dtype=torch.int32) + 7
    v, s = dt.mixed(mo, mk, mv)
    for i, (k, op) in enumerate(zip(mk.tolist(), mo.tolist())):
        if op == 0:
            ok &= (int(s[i]) == (1 if k in model else 0)) and (int(s[i]) == 0 or int(v[i]) == model[k])
        elif op == 1:
            ok &= int(s[i]) == (2 if k in model else 1)
        else:
            ok &= int(s[i]) == (1 if k in model else 0)
    for r in range(world):
        for k, op, j in zip(allk[r * 300:(r + 1) * 300], allops[r * 300:(r + 1) * 300], range(300)):
            if op == 1:
                model[int(k)] = j + 7
            elif op == 2:
                model.pop(int(k), None)
    # union of the shards == the single-table model
    sizes = [None] * world
    dist.all_gather_object(sizes, len(dt.shard.m))
    ok &= sum(sizes) == len(model)
    q.put((rank, bool(ok)))
    dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("world,chunks", [(2, 1), (2, 3), (3, 4)])
def test_router_orchestration_gloo(world, chunks):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, chunks)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert res == {r: True for r in range(world)}
