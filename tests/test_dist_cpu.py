"""world_size-2 gloo test of the sharded router's orchestration (DistTable):
count exchange, splits, forward and reverse all-to-all, unpermute.  The per-rank
table is an injected CPU stand-in (a dict with key % world routing); the CUDA
routing kernels are covered by tests/test_gpu_dist.py.  The fused peer-memory
path (DistTable(p2p=True)) runs the same checks with shared-memory stand-ins
for its IPC buffers; its kernels are covered by tests/test_gpu_p2p.py.  No GPU
needed."""
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


# ----------------------------------------------------- peer-memory stand-ins
# The fused routing path (DistTable(p2p=True), PeerRouter) with its CUDA pieces
# replaced: receive / counter / result buffers are POSIX shared memory (a
# handle is the segment name), the counter reservation is a file lock (the
# kernel's atomicAdd_system), and push / reply are numpy loops with the same
# contract as dyc_route_push / dyc_route_reply (SoA receive buffer: keys @0,
# values @4cap, meta @8cap = src_index | src_rank << 32, tags @16cap).
_REG = {}


def _reg(shm):
    pid = len(_REG) + 1
    _REG[pid] = shm
    return pid


class ShmBuffer:
    def __init__(self, nbytes):
        from multiprocessing import shared_memory
        self.shm = shared_memory.SharedMemory(create=True, size=max(8, nbytes))
        self.shm.buf[:] = bytes(self.shm.size)
        self.ptr, self.nbytes, self._opened = _reg(self.shm), nbytes, []

    def handle(self):
        return self.shm.name.encode()

    def open(self, h):
        from multiprocessing import resource_tracker, shared_memory
        s = shared_memory.SharedMemory(name=h.decode())
        resource_tracker.unregister(s._name, "shared_memory")     # the creator unlinks it
        self._opened.append(s)
        return _reg(s)

    def tensor(self, n, dtype, offset=0):
        if n == 0:
            return torch.empty(0, dtype=dtype)
        return torch.frombuffer(self.shm.buf, dtype=dtype, count=n, offset=offset)

    def close(self):
        for s in self._opened:
            s.close()
        self._opened = []
        if self.shm is not None:
            self.shm.close()
            self.shm.unlink()
            self.shm = None


def _np(pid, dtype, count, offset=0):
    return np.frombuffer(_REG[pid].buf, dtype=dtype, count=count, offset=offset)


class DictShardP2P(DictShard):
    def route_push(self, keys, values, world, src_rank, recv_ptrs, count_ptrs, cap, tags=None):
        import fcntl
        k = keys.numpy().view(np.uint32)
        dest = k.astype(np.int64) % world
        for w in range(world):
            idx = np.nonzero(dest == w)[0]
            if idx.size == 0:
                continue
            with open(f"/tmp/dyc_p2p_{_REG[count_ptrs[w]].name}.lock", "a") as lk:
                fcntl.flock(lk, fcntl.LOCK_EX)
                ctr = _np(count_ptrs[w], np.uint64, 1)
                base = int(ctr[0])
                ctr[0] = base + idx.size
                fcntl.flock(lk, fcntl.LOCK_UN)
            ok = idx[base + np.arange(idx.size) < cap]
            pos = base + np.arange(ok.size)
            _np(recv_ptrs[w], np.uint32, cap)[pos] = k[ok]
            if values is not None:
                _np(recv_ptrs[w], np.uint32, cap, 4 * cap)[pos] = values.numpy().view(np.uint32)[ok]
            _np(recv_ptrs[w], np.uint64, cap, 8 * cap)[pos] = ok.astype(np.uint64) | (np.uint64(src_rank) << np.uint64(32))
            if tags is not None:
                _np(recv_ptrs[w], np.uint8, cap, 16 * cap)[pos] = tags.numpy()[ok]

    @staticmethod
    def recv_views(buf, cap, m):
        return buf.tensor(m, torch.int32, 0), buf.tensor(m, torch.int32, 4 * cap), buf.tensor(m, torch.uint8, 16 * cap)

    @staticmethod
    def route_reply(recv_ptr, cap, n, world, vals=None, status=None, out_val_ptrs=None, out_status_ptrs=None):
        meta = _np(recv_ptr, np.uint64, n, 8 * cap)
        src = (meta >> np.uint64(32)).astype(np.int64)
        idx = (meta & np.uint64(0xFFFFFFFF)).astype(np.int64)
        for r in range(world):
            sel = np.nonzero(src == r)[0]
            if sel.size == 0:
                continue
            if vals is not None:
                out = _np(out_val_ptrs[r], np.int32, int(idx[sel].max()) + 1)
                out[idx[sel]] = vals.numpy()[sel]
            if status is not None:
                out = _np(out_status_ptrs[r], np.uint8, int(idx[sel].max()) + 1)
                out[idx[sel]] = status.numpy()[sel]


def _worker(rank, world, port, q, chunks, p2p=False):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icde_lizlhs21_b200.dist import DistTable
    if p2p:
        dt = DistTable(DictShardP2P(), force_route=True, p2p=True, max_ops=300, p2p_buffers=ShmBuffer,
                       p2p_sync=lambda: None)
    else:
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
    if p2p:
        dist.barrier()
        dt.p2p.close()
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


@pytest.mark.parametrize("world", [2, 3])
def test_router_p2p_orchestration_gloo(world):
    """DistTable(p2p=True): push -> barrier -> owner batch in place -> reply ->
    counter reset -> barrier, across real processes, with shared-memory
    stand-ins for the IPC buffers (same checks as the NCCL-path test)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, 1, True)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert res == {r: True for r in range(world)}
