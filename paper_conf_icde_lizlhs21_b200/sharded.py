"""Sharded DyCuckoo through the C ABI (dyc_dist_*, include/dycuckoo.h;
SURVEY §8(b)/(e)): argument marshalling only.

One process per GPU.  The routing (grouping kernels, NCCL grouped send/recv of
counts, requests and replies, the owners' batches, the unpermute) runs inside
libdyc.so; torch.distributed is used for one thing only: broadcasting the
128-byte NCCL unique id from rank 0 (`broadcast_unique_id`).  `local_shards`
> 1 puts several complete shards in this process (virtual shards on one GPU:
the same routing code with the exchange degenerate), which is how the
sharded path is parity-tested on one B200.
"""
from __future__ import annotations

import ctypes as C
from typing import Dict, List, Optional

from . import _lib as L
from .table import Table, _check_u32, _stream_ptr


def _torch():
    import torch
    return torch


def new_unique_id() -> bytes:
    """dyc_dist_get_unique_id: 128 bytes (ncclGetUniqueId; needs no GPU)."""
    buf = C.create_string_buffer(L.DYC_NCCL_UNIQUE_ID_BYTES)
    L.check(L.load_library().dyc_dist_get_unique_id(buf), "dyc_dist_get_unique_id")
    return bytes(buf.raw)


def broadcast_unique_id(group=None) -> Optional[bytes]:
    """Rank 0 of `group` creates the id, every rank returns it (None when the
    world has one rank: no communicator is needed)."""
    import torch.distributed as dist
    if not dist.is_available() or not dist.is_initialized():
        return None
    world = dist.get_world_size(group)
    if world == 1:
        return None
    rank = dist.get_rank(group)
    obj: List[Optional[bytes]] = [new_unique_id() if rank == 0 else None]
    src = dist.get_global_rank(group, 0) if group is not None else 0
    dist.broadcast_object_list(obj, src=src, group=group)
    return obj[0]


class ShardedTable:
    """This rank's part of a hash-partitioned table (dyc_dist).  Every rank must
    call the same batch methods in the same order; each returns the results of
    the calling rank's ops in request order."""

    def __init__(self, d: int = 4, init_capacity: int = 1 << 20, alpha: float = 0.3, beta: float = 0.85,
                 bucket_slots: int = 8, seed: int = 0x5EED0001, max_hops: int = 64, local_shards: int = 1,
                 group=None, rank: Optional[int] = None, world: Optional[int] = None,
                 unique_id: Optional[bytes] = None):
        torch = _torch()
        self._lib = L.load_library()
        if rank is None or world is None:
            import torch.distributed as dist
            if dist.is_available() and dist.is_initialized():
                rank, world = dist.get_rank(group), dist.get_world_size(group)
            else:
                rank, world = 0, 1
        if unique_id is None and world > 1:
            unique_id = broadcast_unique_id(group)
        self.rank, self.world, self.local_shards = int(rank), int(world), int(local_shards)
        self.d, self.B = d, bucket_slots
        cfg = L.dyc_config()
        L.check(self._lib.dyc_config_default(C.byref(cfg)), "dyc_config_default")
        cfg.d, cfg.bucket_slots, cfg.alpha, cfg.beta = d, bucket_slots, alpha, beta
        cfg.init_capacity, cfg.seed, cfg.max_hops = init_capacity, seed, max_hops
        h = C.c_void_p()
        uid = C.create_string_buffer(unique_id, L.DYC_NCCL_UNIQUE_ID_BYTES) if unique_id else None
        L.check(self._lib.dyc_dist_create_ex(C.byref(cfg), uid, self.rank, self.world, self.local_shards,
                                             C.byref(h)), "dyc_dist_create_ex")
        self._h = h
        self.device = torch.device("cuda", torch.cuda.current_device())

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            self._lib.dyc_dist_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass

    # ------------------------------------------------------------ batches
    def insert(self, keys, values, status=None, stream=None):
        torch = _torch()
        _check_u32(keys, "keys")
        _check_u32(values, "values")
        n = keys.numel()
        status = torch.empty(n, dtype=torch.uint8, device=keys.device) if status is None else status
        L.check(self._lib.dyc_dist_insert_batch(self._h, keys.data_ptr() or None, values.data_ptr() or None,
                                                status.data_ptr() if n else None, n, _stream_ptr(stream)),
                "dyc_dist_insert_batch")
        return status

    def find(self, keys, stream=None):
        torch = _torch()
        _check_u32(keys, "keys")
        n = keys.numel()
        v = torch.empty(n, dtype=torch.int32, device=keys.device)
        f = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyc_dist_find_batch(self._h, keys.data_ptr() or None, v.data_ptr() if n else None,
                                              f.data_ptr() if n else None, n, _stream_ptr(stream)),
                "dyc_dist_find_batch")
        return v, f

    def delete(self, keys, stream=None):
        torch = _torch()
        _check_u32(keys, "keys")
        n = keys.numel()
        v = torch.empty(n, dtype=torch.int32, device=keys.device)
        s = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyc_dist_delete_batch(self._h, keys.data_ptr() or None, v.data_ptr() if n else None,
                                                s.data_ptr() if n else None, n, _stream_ptr(stream)),
                "dyc_dist_delete_batch")
        return v, s

    def mixed(self, ops, keys, values, stream=None):
        torch = _torch()
        _check_u32(keys, "keys")
        _check_u32(values, "values")
        n = keys.numel()
        v = torch.empty(n, dtype=torch.int32, device=keys.device)
        s = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyc_dist_mixed_batch(self._h, ops.data_ptr() or None, keys.data_ptr() or None,
                                               values.data_ptr() or None, v.data_ptr() if n else None,
                                               s.data_ptr() if n else None, n, _stream_ptr(stream)),
                "dyc_dist_mixed_batch")
        return v, s

    # ------------------------------------------------------------ inspection
    @property
    def last_recv(self) -> int:
        """Ops this rank's shards executed in the last batch."""
        n = C.c_uint64()
        L.check(self._lib.dyc_dist_info(self._h, None, None, None, C.byref(n)), "dyc_dist_info")
        return int(n.value)

    def shard(self, local_index: int) -> Table:
        """Non-owning Table view of local shard `local_index` (stats, dump)."""
        h = C.c_void_p()
        L.check(self._lib.dyc_dist_shard(self._h, local_index, C.byref(h)), "dyc_dist_shard")
        return Table.borrow(h.value, self.d, self.B)

    def clear(self, stream=None) -> None:
        for i in range(self.local_shards):
            self.shard(i).clear(stream)

    def profile(self, enable: bool = True) -> None:
        for i in range(self.local_shards):
            self.shard(i).profile(enable)

    def profile_read(self) -> Dict[str, tuple]:
        """Per-kernel (ms, launches) summed over the local shards."""
        tot: Dict[str, list] = {}
        for i in range(self.local_shards):
            for k, (ms, calls) in self.shard(i).profile_read().items():
                t = tot.setdefault(k, [0.0, 0])
                t[0] += ms
                t[1] += calls
        return {k: (v[0], v[1]) for k, v in tot.items()}

    def launch_count(self, reset: bool = False) -> int:
        return sum(self.shard(i).launch_count(reset=reset) for i in range(self.local_shards))

    def stats(self) -> List[Dict]:
        return [self.shard(i).stats() for i in range(self.local_shards)]

    def sorted_kv(self):
        """Union of the local shards' contents, sorted by key (tests)."""
        import numpy as np
        kv = np.concatenate([self.shard(i).dump()[0] for i in range(self.local_shards)])
        keys = (kv & np.uint64(0xFFFFFFFF)).astype(np.uint32)
        return kv[np.argsort(keys, kind="stable")]
