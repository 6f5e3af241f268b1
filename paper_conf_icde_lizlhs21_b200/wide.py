"""Python view of the wide-key table (include/dycuckoo_wide.h).

Keys are CUDA tensors of dtype torch.int64 / torch.uint64 (reinterpreted as
uint64; -1 == 0xFFFF_FFFF_FFFF_FFFF is the reserved EMPTY key); values are
int64 tensors of shape (n, W).  Argument marshalling only: every step runs in
the CUDA kernels of libdyc.so.
"""
from __future__ import annotations

import ctypes as C
from typing import Dict, Tuple

import numpy as np

from . import _lib as L
from .table import _stream_ptr, _torch

MODES = {"voter": L.DYW_MODE_VOTER, "grouped": L.DYW_MODE_GROUPED, "lockfree": L.DYW_MODE_LOCKFREE}


def _check_u64(t, name, ndim=1):
    torch = _torch()
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor")
    if t.dtype not in (torch.int64, torch.uint64):
        raise TypeError(f"{name} must be int64/uint64, got {t.dtype}")
    if not t.is_contiguous() or t.dim() != ndim:
        raise ValueError(f"{name} must be contiguous with {ndim} dimension(s)")


class WideTable:
    """A wide-key DyCuckoo table: u64 keys, W-word values, one of three
    placement modes ("voter" = Alg. 1 bucket locks, "grouped" = per-lane
    try-locks, "lockfree" = 128-bit atomics, W = 1)."""

    def __init__(self, d: int = 4, init_capacity: int = 4096, alpha: float = 0.3, beta: float = 0.85,
                 value_words: int = 2, mode: str = "voter", seed: int = 0x5EED0001, max_hops: int = 64):
        self._lib = L.load_library()
        cfg = L.dyw_config()
        L.check(self._lib.dyw_config_default(C.byref(cfg)), "dyw_config_default")
        cfg.d, cfg.value_words, cfg.mode, cfg.max_hops = d, value_words, MODES[mode], max_hops
        cfg.alpha, cfg.beta, cfg.init_capacity, cfg.seed = alpha, beta, init_capacity, seed
        h = C.c_void_p()
        L.check(self._lib.dyw_create(C.byref(cfg), C.byref(h)), "dyw_create")
        self._h = h
        self.d, self.W, self.mode = d, value_words, mode

    def close(self):
        if getattr(self, "_h", None):
            self._lib.dyw_destroy(self._h)
            self._h = None

    __del__ = close

    def insert(self, keys, values, status=None, stream=None):
        torch = _torch()
        _check_u64(keys, "keys")
        _check_u64(values, "values", 2)
        n = keys.numel()
        if values.shape != (n, self.W):
            raise ValueError(f"values must have shape ({n}, {self.W})")
        if status is None:
            status = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyw_insert_batch(self._h, keys.data_ptr(), values.data_ptr(), status.data_ptr() if n else None,
                                           n, _stream_ptr(stream)), "dyw_insert_batch")
        return status

    def find(self, keys, values_out=None, found=None, stream=None):
        torch = _torch()
        _check_u64(keys, "keys")
        n = keys.numel()
        if values_out is None:
            values_out = torch.empty((n, self.W), dtype=torch.int64, device=keys.device)
        if found is None:
            found = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyw_find_batch(self._h, keys.data_ptr(), values_out.data_ptr(), found.data_ptr() if n else None,
                                         n, _stream_ptr(stream)), "dyw_find_batch")
        return values_out, found

    def delete(self, keys, values_out=None, status=None, stream=None):
        torch = _torch()
        _check_u64(keys, "keys")
        n = keys.numel()
        if values_out is None:
            values_out = torch.empty((n, self.W), dtype=torch.int64, device=keys.device)
        if status is None:
            status = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyw_delete_batch(self._h, keys.data_ptr(), values_out.data_ptr(),
                                           status.data_ptr() if n else None, n, _stream_ptr(stream)),
                "dyw_delete_batch")
        return values_out, status

    def resize(self, direction: int, subtable: int = -1, stream=None):
        L.check(self._lib.dyw_resize(self._h, direction, subtable, _stream_ptr(stream)), "dyw_resize")

    def clear(self, stream=None):
        L.check(self._lib.dyw_clear(self._h, _stream_ptr(stream)), "dyw_clear")

    def stats(self, stream=None) -> Dict:
        s = L.dyw_stats_t()
        L.check(self._lib.dyw_stats(self._h, C.byref(s), _stream_ptr(stream)), "dyw_stats")
        d = s.d
        return dict(m=s.m, N=s.N, d=d, B=s.B, W=s.W, mode=s.mode, buckets=list(s.buckets[:d]),
                    count=list(s.count[:d]), fill=s.fill, n_upsize=s.n_upsize, n_downsize=s.n_downsize,
                    n_fail_upsize=s.n_fail_upsize, n_residual=s.n_residual, n_evict=s.n_evict,
                    n_lock_fail=s.n_lock_fail, last_insert_new=s.last_insert_new,
                    last_insert_pending=s.last_insert_pending, bytes_allocated=s.bytes_allocated)

    def dump(self, stream=None):
        """(keys u64, values u64 (m, W), table u32, bucket u64) host arrays, any order."""
        m = self.stats(stream)["m"]
        k = np.empty(m, dtype=np.uint64)
        v = np.empty((m, self.W), dtype=np.uint64)
        tb = np.empty(m, dtype=np.uint32)
        bk = np.empty(m, dtype=np.uint64)
        n = C.c_uint64()
        L.check(self._lib.dyw_dump(self._h, k.ctypes.data, v.ctypes.data, tb.ctypes.data, bk.ctypes.data, m,
                                   C.byref(n), _stream_ptr(stream)), "dyw_dump")
        return k, v, tb, bk

    def sorted_items(self) -> Tuple[np.ndarray, np.ndarray]:
        k, v, _, _ = self.dump()
        o = np.argsort(k, kind="stable")
        return k[o], v[o]

    def hash_probe(self, keys):
        torch = _torch()
        _check_u64(keys, "keys")
        n = keys.numel()
        x = torch.empty((n, self.d + 2), dtype=torch.int32, device=keys.device)
        p = torch.empty((n, 2), dtype=torch.int32, device=keys.device)
        L.check(self._lib.dyw_hash_probe(self._h, keys.data_ptr(), n, x.data_ptr(), p.data_ptr(),
                                         _stream_ptr(None)), "dyw_hash_probe")
        return x, p

    def launch_count(self, reset: bool = False) -> int:
        return int(self._lib.dyw_launch_count(self._h, 1 if reset else 0))
