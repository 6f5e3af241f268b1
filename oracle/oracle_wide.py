"""ctypes wrapper around oracle/dyw_oracle.c, the wide-key oracle (NEXT-3).

TEST INFRASTRUCTURE ONLY.  Argument marshalling only: every step runs in the
plain C file.  Keys are uint64 (0xFFFF_FFFF_FFFF_FFFF reserved), values are W
uint64 words per key (arrays of shape (n, W)).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from typing import Dict, Optional, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "dyw_oracle.c")
_LIB = os.path.join(_HERE, "libdyw_oracle.so")
DMAX = 16
EMPTY64 = 0xFFFFFFFFFFFFFFFF


class _Stats(C.Structure):
    _fields_ = [
        ("m", C.c_uint64), ("N", C.c_uint64), ("d", C.c_uint32), ("B", C.c_uint32),
        ("W", C.c_uint32), ("pad", C.c_uint32),
        ("buckets", C.c_uint64 * DMAX), ("count", C.c_uint64 * DMAX),
        ("n_upsize", C.c_uint64), ("n_downsize", C.c_uint64), ("n_fail_upsize", C.c_uint64),
        ("n_residual", C.c_uint64), ("n_evict", C.c_uint64),
        ("max_probes", C.c_uint64), ("invariant_errors", C.c_uint64),
    ]


def build_oracle_wide(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def oracle_wide_lib():
    global _lib
    if _lib is None:
        lib = C.CDLL(build_oracle_wide())
        P, U32, U64, I32, D = C.c_void_p, C.c_uint32, C.c_uint64, C.c_int, C.c_double
        lib.dyw_o_create.restype = P
        lib.dyw_o_create.argtypes = [U32, U32, U32, U64, D, D, U64, U32]
        lib.dyw_o_destroy.argtypes = [P]
        for name in ("dyw_o_insert_batch", "dyw_o_find_batch", "dyw_o_delete_batch"):
            getattr(lib, name).argtypes = [P, P, P, P, U64]
        lib.dyw_o_resize.argtypes = [P, I32, I32]
        lib.dyw_o_resize.restype = I32
        lib.dyw_o_stats.argtypes = [P, C.POINTER(_Stats)]
        lib.dyw_o_dump.argtypes = [P, P, P, P, P, U64]
        lib.dyw_o_dump.restype = U64
        lib.dyw_o_check_invariants.argtypes = [P, C.c_char_p, U64]
        lib.dyw_o_check_invariants.restype = U64
        lib.dyw_o_hash_x.argtypes = [P, U32, U64]
        lib.dyw_o_hash_x.restype = U64
        lib.dyw_o_pair.argtypes = [P, U64, C.POINTER(U32), C.POINTER(U32)]
        lib.dyw_o_bucket.argtypes = [P, U32, U64]
        lib.dyw_o_bucket.restype = U64
        lib.dyw_o_hash_params.argtypes = [P, P, P, P]
        lib.dyw_o_check_layout.argtypes = [P, P, P, P, P, U64]
        lib.dyw_o_check_layout.restype = U64
        _lib = lib
    return _lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


class OracleWideTable:
    """Sequential wide-key DyCuckoo (oracle/dyw_oracle.c)."""

    def __init__(self, d: int = 4, init_capacity: int = 4096, alpha: float = 0.3, beta: float = 0.85,
                 bucket_slots: int = 16, value_words: int = 2, seed: int = 0x5EED0001, max_hops: int = 64):
        self._lib = oracle_wide_lib()
        self.d, self.B, self.W = d, bucket_slots, value_words
        self._t = self._lib.dyw_o_create(d, bucket_slots, value_words, init_capacity, alpha, beta, seed,
                                         max_hops)
        if not self._t:
            raise ValueError("dyw_o_create rejected the arguments")

    def close(self):
        if self._t:
            self._lib.dyw_o_destroy(self._t)
            self._t = None

    __del__ = close

    def _vals(self, values, n):
        v = np.ascontiguousarray(values, dtype=np.uint64).reshape(n, self.W)
        return v

    def insert(self, keys: np.ndarray, values: np.ndarray) -> np.ndarray:
        keys = np.ascontiguousarray(keys, dtype=np.uint64)
        v = self._vals(values, keys.size)
        st = np.zeros(keys.size, dtype=np.uint8)
        self._lib.dyw_o_insert_batch(self._t, _ptr(keys), _ptr(v), _ptr(st), keys.size)
        return st

    def find(self, keys: np.ndarray) -> Tuple[np.ndarray, np.ndarray]:
        keys = np.ascontiguousarray(keys, dtype=np.uint64)
        v = np.zeros((keys.size, self.W), dtype=np.uint64)
        f = np.zeros(keys.size, dtype=np.uint8)
        self._lib.dyw_o_find_batch(self._t, _ptr(keys), _ptr(v), _ptr(f), keys.size)
        return v, f

    def delete(self, keys: np.ndarray) -> Tuple[np.ndarray, np.ndarray]:
        keys = np.ascontiguousarray(keys, dtype=np.uint64)
        v = np.zeros((keys.size, self.W), dtype=np.uint64)
        st = np.zeros(keys.size, dtype=np.uint8)
        self._lib.dyw_o_delete_batch(self._t, _ptr(keys), _ptr(v), _ptr(st), keys.size)
        return v, st

    def resize(self, direction: int, subtable: int = -1) -> int:
        return int(self._lib.dyw_o_resize(self._t, direction, subtable))

    def stats(self) -> Dict:
        s = _Stats()
        self._lib.dyw_o_stats(self._t, C.byref(s))
        d = s.d
        return dict(m=s.m, N=s.N, d=d, B=s.B, W=s.W, buckets=list(s.buckets[:d]), count=list(s.count[:d]),
                    n_upsize=s.n_upsize, n_downsize=s.n_downsize, n_fail_upsize=s.n_fail_upsize,
                    n_residual=s.n_residual, n_evict=s.n_evict, max_probes=s.max_probes,
                    invariant_errors=s.invariant_errors, fill=(s.m / s.N) if s.N else 0.0)

    def dump(self):
        n = int(self._lib.dyw_o_dump(self._t, None, None, None, None, 0))
        k = np.zeros(n, dtype=np.uint64)
        v = np.zeros((n, self.W), dtype=np.uint64)
        tb = np.zeros(n, dtype=np.uint32)
        bk = np.zeros(n, dtype=np.uint64)
        self._lib.dyw_o_dump(self._t, _ptr(k), _ptr(v), _ptr(tb), _ptr(bk), n)
        return k, v, tb, bk

    def sorted_items(self) -> Tuple[np.ndarray, np.ndarray]:
        k, v, _, _ = self.dump()
        o = np.argsort(k, kind="stable")
        return k[o], v[o]

    def check_invariants(self) -> Tuple[int, str]:
        buf = C.create_string_buffer(256)
        bad = int(self._lib.dyw_o_check_invariants(self._t, buf, 256))
        return bad, buf.value.decode()

    def check_layout(self, buckets, keys, tables, bucket_idx) -> int:
        nb = np.ascontiguousarray(buckets, dtype=np.uint64)
        keys = np.ascontiguousarray(keys, dtype=np.uint64)
        tables = np.ascontiguousarray(tables, dtype=np.uint32)
        bucket_idx = np.ascontiguousarray(bucket_idx, dtype=np.uint64)
        return int(self._lib.dyw_o_check_layout(self._t, _ptr(nb), _ptr(keys), _ptr(tables), _ptr(bucket_idx),
                                                keys.size))

    def hash_x(self, s: int, k: int) -> int:
        return int(self._lib.dyw_o_hash_x(self._t, s, k))

    def pair(self, k: int) -> Tuple[int, int]:
        a, b = C.c_uint32(), C.c_uint32()
        self._lib.dyw_o_pair(self._t, k, C.byref(a), C.byref(b))
        return a.value, b.value

    def bucket(self, t: int, k: int) -> int:
        return int(self._lib.dyw_o_bucket(self._t, t, k))

    def hash_params(self):
        a = np.zeros(self.d + 2, dtype=np.uint64)
        b = np.zeros(self.d + 2, dtype=np.uint64)
        c = np.zeros(self.d + 2, dtype=np.uint64)
        self._lib.dyw_o_hash_params(self._t, _ptr(a), _ptr(b), _ptr(c))
        return a, b, c
