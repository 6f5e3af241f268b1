"""Python view of a libdyc.so table.  PyTorch supplies device memory and streams
only; every step of the hot path runs in the CUDA kernels behind the C ABI.

Keys/values are passed as CUDA tensors of dtype torch.int32 or torch.uint32
(reinterpreted as uint32; element i is op i).  Status/found arrays are uint8.
"""
from __future__ import annotations

import ctypes as C
from typing import Dict, Optional, Tuple

import numpy as np

from . import _lib as L

_U32_DTYPES = None


def _torch():
    import torch
    return torch


def _check_u32(t, name):
    torch = _torch()
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor")
    if t.dtype not in (torch.int32, torch.uint32):
        raise TypeError(f"{name} must be int32/uint32, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")


def _stream_ptr(stream) -> int:
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream()
    return int(s.cuda_stream)


def _ptr_array(ptrs, world: int):
    if len(ptrs) != world:
        raise ValueError(f"expected {world} device pointers, got {len(ptrs)}")
    return C.cast((C.c_void_p * world)(*[int(p) for p in ptrs]), C.c_void_p)


class PeerBuffer:
    """A device buffer from dyc_ipc_alloc (plain cudaMalloc, zero-filled) that
    other processes map through CUDA IPC (dyc_ipc_get_handle / dyc_ipc_open).
    `ptr` is the local address; `handle()` the 64-byte IPC handle; `open(h)`
    maps a peer's handle and returns its address here (closed by close())."""

    def __init__(self, nbytes: int):
        p = C.c_void_p()
        L.check(L.load_library().dyc_ipc_alloc(int(nbytes), C.byref(p)), "dyc_ipc_alloc")
        self.ptr, self.nbytes, self._opened = int(p.value), int(nbytes), []

    def handle(self) -> bytes:
        h = (C.c_char * 64)()
        L.check(L.load_library().dyc_ipc_get_handle(self.ptr, h), "dyc_ipc_get_handle")
        return bytes(h.raw)

    def open(self, handle: bytes) -> int:
        p = C.c_void_p()
        L.check(L.load_library().dyc_ipc_open(C.create_string_buffer(handle, 64), C.byref(p)), "dyc_ipc_open")
        self._opened.append(int(p.value))
        return int(p.value)

    def tensor(self, n: int, dtype, offset: int = 0):
        """Zero-copy torch view of n elements at byte `offset` (__cuda_array_interface__)."""
        torch = _torch()
        typestr = {torch.int32: "<i4", torch.uint8: "|u1", torch.int64: "<i8"}[dtype]
        size = n * torch.tensor([], dtype=dtype).element_size()
        if offset + size > self.nbytes:
            raise ValueError("view outside the buffer")
        if n == 0:
            return torch.empty(0, dtype=dtype, device="cuda")
        ptr = self.ptr + offset

        class _View:
            __cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3,
                                        "strides": None, "stream": None}
        return torch.as_tensor(_View(), device="cuda")

    def close(self):
        lib = L.load_library()
        for p in self._opened:
            lib.dyc_ipc_close(p)
        self._opened = []
        if self.ptr:
            lib.dyc_ipc_free(self.ptr)
            self.ptr = 0

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass


class Table:
    """A DyCuckoo table (two-layer cuckoo hash, d subtables; see include/dycuckoo.h)."""

    def __init__(self, d: int = 4, init_capacity: int = 4096, alpha: float = 0.3, beta: float = 0.85,
                 bucket_slots: int = 8, seed: int = 0x5EED0001, max_hops: int = 64, device=None,
                 placement: str = "first_fit", in_place: bool = False, staged: str = "auto"):
        torch = _torch()
        self._lib = L.load_library()
        if not torch.cuda.is_available():
            raise RuntimeError("dycuckoo needs a CUDA device (no CPU fallback)")
        self.device = torch.device("cuda", torch.cuda.current_device() if device is None else
                                   torch.device(device).index or 0)
        cfg = L.dyc_config()
        L.check(self._lib.dyc_config_default(C.byref(cfg)), "dyc_config_default")
        cfg.d, cfg.bucket_slots, cfg.alpha, cfg.beta = d, bucket_slots, alpha, beta
        cfg.init_capacity, cfg.seed, cfg.max_hops = init_capacity, seed, max_hops
        if placement not in ("first_fit", "paper_weighted"):
            raise ValueError("placement must be 'first_fit' (reading Q3) or 'paper_weighted' (P:L361)")
        cfg.flags = (cfg.flags & ~L.DYC_PLACE_PAPER_WEIGHTED) | (
            L.DYC_PLACE_PAPER_WEIGHTED if placement == "paper_weighted" else 0)
        cfg.flags = (cfg.flags & ~L.DYC_RESIZE_IN_PLACE) | (L.DYC_RESIZE_IN_PLACE if in_place else 0)
        if staged not in ("auto", "off", "force"):
            raise ValueError("staged must be 'auto', 'off' or 'force' (DYC_STAGED_*)")
        cfg.flags |= {"auto": 0, "off": L.DYC_STAGED_OFF, "force": L.DYC_STAGED_FORCE}[staged]
        self.placement = placement
        self.cfg = cfg
        h = C.c_void_p()
        with torch.cuda.device(self.device):
            L.check(self._lib.dyc_create_ex(C.byref(cfg), C.byref(h)), "dyc_create_ex")
        self._h = h
        self.d, self.B = d, bucket_slots

    @property
    def handle(self) -> int:
        return self._h.value

    @classmethod
    def borrow(cls, handle: int, d: int, bucket_slots: int) -> "Table":
        """A non-owning view of a table owned elsewhere (a shard of a dyc_dist):
        stats / dump / find work on it; close() does not destroy it."""
        torch = _torch()
        t = cls.__new__(cls)
        t._lib = L.load_library()
        t.device = torch.device("cuda", torch.cuda.current_device())
        t._h = C.c_void_p(handle)
        t.d, t.B = d, bucket_slots
        t._borrowed = True
        return t

    def close(self):
        if getattr(self, "_borrowed", False):
            self._h = C.c_void_p()
            return
        if getattr(self, "_h", None) is not None and self._h.value:
            self._lib.dyc_destroy(self._h)
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
        if values.numel() != n:
            raise ValueError("keys/values length mismatch")
        if status is None:
            status = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyc_insert_batch(self._h, keys.data_ptr(), values.data_ptr(),
                                           status.data_ptr() if n else None, n, _stream_ptr(stream)),
                "dyc_insert_batch")
        return status

    def find(self, keys, values_out=None, found=None, stream=None):
        torch = _torch()
        _check_u32(keys, "keys")
        n = keys.numel()
        if values_out is None:
            values_out = torch.empty(n, dtype=torch.int32, device=keys.device)
        if found is None:
            found = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyc_find_batch(self._h, keys.data_ptr(), values_out.data_ptr(),
                                         found.data_ptr() if n else None, n, _stream_ptr(stream)),
                "dyc_find_batch")
        return values_out, found

    def delete(self, keys, values_out=None, status=None, stream=None, want_values=True):
        torch = _torch()
        _check_u32(keys, "keys")
        n = keys.numel()
        if values_out is None and want_values:
            values_out = torch.empty(n, dtype=torch.int32, device=keys.device)
        if status is None:
            status = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyc_delete_batch(self._h, keys.data_ptr(),
                                           values_out.data_ptr() if (values_out is not None and n) else None,
                                           status.data_ptr() if n else None, n, _stream_ptr(stream)),
                "dyc_delete_batch")
        return values_out, status

    # one batch delivered in parts (dyc_*_begin / _part / _end)
    def insert_begin(self, n_total: int, stream=None):
        L.check(self._lib.dyc_insert_begin(self._h, n_total, _stream_ptr(stream)), "dyc_insert_begin")

    def insert_part(self, keys, values, status=None, stream=None):
        torch = _torch()
        n = keys.numel()
        if status is None:
            status = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyc_insert_part(self._h, keys.data_ptr() if n else None, values.data_ptr() if n else None,
                                          status.data_ptr() if n else None, n, _stream_ptr(stream)),
                "dyc_insert_part")
        return status

    def insert_end(self, stream=None):
        L.check(self._lib.dyc_insert_end(self._h, _stream_ptr(stream)), "dyc_insert_end")

    def delete_begin(self, n_total: int, stream=None):
        L.check(self._lib.dyc_delete_begin(self._h, n_total, _stream_ptr(stream)), "dyc_delete_begin")

    def delete_part(self, keys, values_out=None, status=None, stream=None):
        torch = _torch()
        n = keys.numel()
        if values_out is None:
            values_out = torch.empty(n, dtype=torch.int32, device=keys.device)
        if status is None:
            status = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyc_delete_part(self._h, keys.data_ptr() if n else None,
                                          values_out.data_ptr() if n else None, status.data_ptr() if n else None,
                                          n, _stream_ptr(stream)), "dyc_delete_part")
        return values_out, status

    def delete_end(self, stream=None):
        L.check(self._lib.dyc_delete_end(self._h, _stream_ptr(stream)), "dyc_delete_end")

    def mixed(self, ops, keys, values, values_out=None, status=None, stream=None):
        """Mixed batch (find=0, insert=1, delete=2; phases find -> insert -> delete, Q10)."""
        torch = _torch()
        _check_u32(keys, "keys")
        _check_u32(values, "values")
        n = keys.numel()
        if values_out is None:
            values_out = torch.empty(n, dtype=torch.int32, device=keys.device)
        if status is None:
            status = torch.empty(n, dtype=torch.uint8, device=keys.device)
        L.check(self._lib.dyc_mixed_batch(self._h, ops.data_ptr(), keys.data_ptr(), values.data_ptr(),
                                          values_out.data_ptr(), status.data_ptr(), n, _stream_ptr(stream)),
                "dyc_mixed_batch")
        return values_out, status

    # host-buffer entry points (end-to-end path: copies inside the call, chunked
    # so PCIe transfers overlap the kernels).  Output arrays may be supplied
    # (e.g. pinned numpy views) to avoid pageable-memory copies.
    def insert_host(self, keys: np.ndarray, values: np.ndarray, status: Optional[np.ndarray] = None,
                    stream=None) -> np.ndarray:
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        values = np.ascontiguousarray(values, dtype=np.uint32)
        st = np.empty(keys.size, dtype=np.uint8) if status is None else status
        L.check(self._lib.dyc_insert_batch_host(self._h, keys.ctypes.data, values.ctypes.data, st.ctypes.data,
                                                keys.size, _stream_ptr(stream)), "dyc_insert_batch_host")
        return st

    def find_host(self, keys: np.ndarray, values_out: Optional[np.ndarray] = None,
                  found: Optional[np.ndarray] = None, stream=None) -> Tuple[np.ndarray, np.ndarray]:
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        v = np.empty(keys.size, dtype=np.uint32) if values_out is None else values_out
        f = np.empty(keys.size, dtype=np.uint8) if found is None else found
        L.check(self._lib.dyc_find_batch_host(self._h, keys.ctypes.data, v.ctypes.data, f.ctypes.data,
                                              keys.size, _stream_ptr(stream)), "dyc_find_batch_host")
        return v, f

    def delete_host(self, keys: np.ndarray, values_out: Optional[np.ndarray] = None,
                    status: Optional[np.ndarray] = None, stream=None) -> Tuple[np.ndarray, np.ndarray]:
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        v = np.empty(keys.size, dtype=np.uint32) if values_out is None else values_out
        s = np.empty(keys.size, dtype=np.uint8) if status is None else status
        L.check(self._lib.dyc_delete_batch_host(self._h, keys.ctypes.data, v.ctypes.data, s.ctypes.data,
                                                keys.size, _stream_ptr(stream)), "dyc_delete_batch_host")
        return v, s

    # ------------------------------------------------------------ control
    def resize(self, direction: int, subtable: int = -1, method: int = L.DYC_RESIZE_SPLIT, stream=None):
        L.check(self._lib.dyc_resize_ex(self._h, direction, subtable, method, _stream_ptr(stream)),
                "dyc_resize_ex")

    def resize_begin(self, direction: int, subtable: int = -1, stream=None, resize_stream=None):
        """Start a one-subtable resize on `resize_stream` and return at once
        (dyc_resize_begin; NEXT-1).  Batches issued on `stream`
        before dyc_resize_commit run concurrently with it."""
        if resize_stream is None:
            raise ValueError("resize_begin needs a resize_stream (a torch.cuda.Stream)")
        L.check(self._lib.dyc_resize_begin(self._h, direction, subtable, _stream_ptr(stream),
                                           _stream_ptr(resize_stream)), "dyc_resize_begin")

    def resize_commit(self, stream=None):
        L.check(self._lib.dyc_resize_commit(self._h, _stream_ptr(stream)), "dyc_resize_commit")

    def resize_query(self):
        """(in_flight, kernel_done) of the resize started by resize_begin."""
        a, b = C.c_int(), C.c_int()
        L.check(self._lib.dyc_resize_query(self._h, C.byref(a), C.byref(b)), "dyc_resize_query")
        return bool(a.value), bool(b.value)

    def trim(self):
        """Return cached (released) device buffers to the device."""
        L.check(self._lib.dyc_trim(self._h), "dyc_trim")

    def clear(self, stream=None):
        L.check(self._lib.dyc_clear(self._h, _stream_ptr(stream)), "dyc_clear")

    def shape(self) -> Dict:
        """Host view without touching the device (dyc_shape: never synchronizes):
        buckets per subtable, the live-count bounds m_lo <= m <= m_hi left by
        batches that skipped their read-back, failure-triggered upsizes so far."""
        nb = np.zeros(self.d, dtype=np.uint64)
        lo, hi, nf = C.c_uint64(), C.c_uint64(), C.c_uint64()
        L.check(self._lib.dyc_shape(self._h, nb.ctypes.data_as(C.c_void_p), C.byref(lo), C.byref(hi), C.byref(nf)),
                "dyc_shape")
        return {"buckets": [int(x) for x in nb], "m_lo": int(lo.value), "m_hi": int(hi.value),
                "n_fail_upsize": int(nf.value)}

    def _buckets_host(self):
        return self.shape()["buckets"]

    def stats(self, stream=None) -> Dict:
        s = L.dyc_stats_t()
        L.check(self._lib.dyc_stats(self._h, C.byref(s), _stream_ptr(stream)), "dyc_stats")
        d = s.d
        return dict(m=s.m, N=s.N, d=d, B=s.B, buckets=list(s.buckets[:d]), count=list(s.count[:d]),
                    fill=s.fill, n_upsize=s.n_upsize, n_downsize=s.n_downsize,
                    n_fail_upsize=s.n_fail_upsize, n_residual=s.n_residual, n_evict=s.n_evict,
                    n_place_retry=s.n_place_retry, n_second_table=s.n_second_table,
                    bytes_allocated=s.bytes_allocated, last_insert_new=s.last_insert_new,
                    last_insert_pending=s.last_insert_pending,
                    last_insert_evictions=s.last_insert_evictions, bytes_cached=s.bytes_cached,
                    n_live_resize=s.n_live_resize, n_deferred=s.n_deferred,
                    n_device_alloc=s.n_device_alloc, alloc_ms=s.alloc_ms, n_sync=s.n_sync, sync_ms=s.sync_ms,
                    n_pending=s.n_pending, vm_subtables=s.vm_subtables, vm_mapped_bytes=s.vm_mapped_bytes,
                    n_vm_map=s.n_vm_map, n_vm_unmap=s.n_vm_unmap, n_staged=s.n_staged)

    def dump(self, stream=None):
        """(kv uint64, table uint32, bucket uint64) host arrays, unspecified order."""
        n = C.c_uint64()
        st = self.stats(stream)
        m = st["m"]
        kv = np.empty(m, dtype=np.uint64)
        tb = np.empty(m, dtype=np.uint32)
        bk = np.empty(m, dtype=np.uint64)
        L.check(self._lib.dyc_dump(self._h, kv.ctypes.data, tb.ctypes.data, bk.ctypes.data, m, C.byref(n),
                                   _stream_ptr(stream)), "dyc_dump")
        return kv, tb, bk

    def sorted_kv(self, stream=None) -> np.ndarray:
        kv, _, _ = self.dump(stream)
        keys = (kv & np.uint64(0xFFFFFFFF)).astype(np.uint32)
        return kv[np.argsort(keys, kind="stable")]

    def hash_params(self) -> Tuple[np.ndarray, np.ndarray]:
        a = np.zeros(self.d + 2, dtype=np.uint64)
        b = np.zeros(self.d + 2, dtype=np.uint64)
        L.check(self._lib.dyc_hash_params(self._h, a.ctypes.data, b.ctypes.data), "dyc_hash_params")
        return a, b

    def hash_probe(self, keys, stream=None):
        torch = _torch()
        _check_u32(keys, "keys")
        n = keys.numel()
        x = torch.empty(n * (self.d + 2), dtype=torch.int32, device=keys.device)
        pr = torch.empty(2 * n, dtype=torch.int32, device=keys.device)
        L.check(self._lib.dyc_hash_probe(self._h, keys.data_ptr(), n, x.data_ptr(), pr.data_ptr(),
                                         _stream_ptr(stream)), "dyc_hash_probe")
        return x.view(n, self.d + 2), pr.view(n, 2)

    def profile(self, enable: bool = True) -> None:
        L.check(self._lib.dyc_profile_enable(self._h, 1 if enable else 0), "dyc_profile_enable")

    def profile_read(self) -> Dict[str, Tuple[float, int]]:
        ms = np.zeros(L.DYC_PROF_KINDS, dtype=np.float64)
        calls = np.zeros(L.DYC_PROF_KINDS, dtype=np.uint64)
        L.check(self._lib.dyc_profile_read(self._h, ms.ctypes.data, calls.ctypes.data), "dyc_profile_read")
        return {name: (float(ms[i]), int(calls[i])) for i, name in enumerate(L.PROF_NAMES)}

    def probe_count(self, enable: bool = True) -> None:
        """Count ops and second-bucket probes in k_find / k_upsert / k_delete (measurement)."""
        L.check(self._lib.dyc_probe_count_enable(self._h, 1 if enable else 0), "dyc_probe_count_enable")

    def probe_count_read(self) -> Dict[str, Tuple[int, int]]:
        """{kind: (ops, second probes)} since the last read; resets the counts."""
        out = np.zeros(6, dtype=np.uint64)
        L.check(self._lib.dyc_probe_count_read(self._h, out.ctypes.data), "dyc_probe_count_read")
        return {k: (int(out[2 * i]), int(out[2 * i + 1])) for i, k in enumerate(("find", "upsert", "delete"))}

    def clean_mask(self) -> int:
        """Bit t: subtable t holds the first-choice-full invariant (dyc_clean_mask)."""
        m = C.c_uint32()
        L.check(self._lib.dyc_clean_mask(self._h, C.byref(m)), "dyc_clean_mask")
        return int(m.value)

    # ------------------------------------------------------------ routing (S11)
    def route_count(self, keys, world: int, counts=None, stream=None):
        """Per-shard histogram (uint64 -> int64 tensor of length world)."""
        torch = _torch()
        _check_u32(keys, "keys")
        if counts is None:
            counts = torch.empty(world, dtype=torch.int64, device=keys.device)
        L.check(self._lib.dyc_route_count(self._h, keys.data_ptr(), keys.numel(), world, counts.data_ptr(),
                                          _stream_ptr(stream)), "dyc_route_count")
        return counts

    def route_scatter(self, keys, values, world: int, counts, stream=None, tags=None):
        """Groups ops by destination shard; returns (keys_out, values_out|None, pos)
        or, with a uint8 `tags` tensor, (keys_out, values_out|None, pos, tags_out)."""
        torch = _torch()
        _check_u32(keys, "keys")
        n = keys.numel()
        kout = torch.empty(n, dtype=torch.int32, device=keys.device)
        vout = torch.empty(n, dtype=torch.int32, device=keys.device) if values is not None else None
        tout = torch.empty(n, dtype=torch.uint8, device=keys.device) if tags is not None else None
        pos = torch.empty(n, dtype=torch.int32, device=keys.device)
        cursor = torch.empty(world, dtype=torch.int64, device=keys.device)
        L.check(self._lib.dyc_route_scatter(self._h, keys.data_ptr(), values.data_ptr() if values is not None else None,
                                            tags.data_ptr() if tags is not None else None, n, world,
                                            counts.data_ptr(), cursor.data_ptr(), kout.data_ptr(),
                                            vout.data_ptr() if vout is not None else None,
                                            tout.data_ptr() if tout is not None else None, pos.data_ptr(),
                                            _stream_ptr(stream)), "dyc_route_scatter")
        return (kout, vout, pos) if tags is None else (kout, vout, pos, tout)

    def route_unpermute(self, pos, reply_vals=None, reply_status=None, stream=None, out_vals=None, out_status=None):
        """vals[i] = reply_vals[pos[i]], status[i] = reply_status[pos[i]] (written
        into out_vals / out_status when given, e.g. slices of the batch result)."""
        torch = _torch()
        n = pos.numel()
        v = s = None
        if reply_vals is not None:
            v = out_vals if out_vals is not None else torch.empty(n, dtype=torch.int32, device=pos.device)
        if reply_status is not None:
            s = out_status if out_status is not None else torch.empty(n, dtype=torch.uint8, device=pos.device)
        L.check(self._lib.dyc_route_unpermute(pos.data_ptr(), n,
                                              reply_vals.data_ptr() if reply_vals is not None else None,
                                              reply_status.data_ptr() if reply_status is not None else None,
                                              v.data_ptr() if v is not None else None,
                                              s.data_ptr() if s is not None else None, _stream_ptr(stream)),
                "dyc_route_unpermute")
        return v, s

    # ------------------------------------------- fused routing over peer memory
    def route_push(self, keys, values, world: int, src_rank: int, recv_ptrs, count_ptrs, recv_cap: int,
                   tags=None, stream=None):
        """Dispatch (dyc_route_push): every op goes to its shard's receive buffer
        (structure-of-arrays, see recv_views).  recv_ptrs / count_ptrs: `world`
        device addresses (ints; peer pointers from PeerBuffer.open or local ones)."""
        _check_u32(keys, "keys")
        L.check(self._lib.dyc_route_push(self._h, keys.data_ptr(), values.data_ptr() if values is not None else None,
                                         tags.data_ptr() if tags is not None else None, keys.numel(), world,
                                         src_rank, _ptr_array(recv_ptrs, world), _ptr_array(count_ptrs, world),
                                         recv_cap, _stream_ptr(stream)), "dyc_route_push")

    @staticmethod
    def recv_views(buf: "PeerBuffer", cap: int, m: int):
        """(keys, values, tags) views of the first m received ops of a receive
        buffer of capacity cap (keys @0, values @4cap, meta @8cap, tags @16cap)."""
        torch = _torch()
        return (buf.tensor(m, torch.int32, 0), buf.tensor(m, torch.int32, 4 * cap),
                buf.tensor(m, torch.uint8, 16 * cap))

    @staticmethod
    def route_reply(recv_ptr: int, recv_cap: int, n: int, world: int, vals=None, status=None, out_val_ptrs=None,
                    out_status_ptrs=None, stream=None):
        """Combine (dyc_route_reply): result j of the receive buffer at recv_ptr
        goes to its requester's result arrays (device addresses per rank)."""
        L.check(L.load_library().dyc_route_reply(
            recv_ptr, recv_cap, n, vals.data_ptr() if vals is not None else None,
            status.data_ptr() if status is not None else None, world,
            _ptr_array(out_val_ptrs, world) if vals is not None else None,
            _ptr_array(out_status_ptrs, world) if status is not None else None,
            _stream_ptr(stream)), "dyc_route_reply")

    def launch_count(self, reset: bool = False) -> int:
        return int(self._lib.dyc_launch_count(self._h, 1 if reset else 0))
