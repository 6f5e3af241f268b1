"""ctypes wrapper around oracle/dyc_oracle.c (TEST INFRASTRUCTURE ONLY).

Argument marshalling only: every step of the oracle runs in the plain C file.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from typing import Dict, Optional, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "dyc_oracle.c")
_LIB = os.path.join(_HERE, "libdyc_oracle.so")
DMAX = 16

FIRST_FIT = 0
PAPER_WEIGHTED = 1


class _Stats(C.Structure):
    _fields_ = [
        ("m", C.c_uint64), ("N", C.c_uint64), ("d", C.c_uint32), ("B", C.c_uint32),
        ("buckets", C.c_uint64 * DMAX), ("count", C.c_uint64 * DMAX),
        ("n_upsize", C.c_uint64), ("n_downsize", C.c_uint64), ("n_fail_upsize", C.c_uint64),
        ("n_residual", C.c_uint64), ("n_evict", C.c_uint64),
        ("max_probes", C.c_uint64), ("n_second_table", C.c_uint64),
        ("invariant_errors", C.c_uint64),
    ]


def build_oracle(force: bool = False) -> str:
    """Compile the plain-C oracle with gcc (no GPU involved)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-shared", "-fPIC",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def oracle_lib():
    global _lib
    if _lib is None:
        lib = C.CDLL(build_oracle())
        P, U32, U64, I32, D = C.c_void_p, C.c_uint32, C.c_uint64, C.c_int, C.c_double
        lib.dyo_create.restype = P
        lib.dyo_create.argtypes = [U32, U32, U64, D, D, U64, U32, U32]
        lib.dyo_destroy.argtypes = [P]
        for name in ("dyo_insert_batch", "dyo_find_batch", "dyo_delete_batch"):
            getattr(lib, name).argtypes = [P, P, P, P, U64]
        lib.dyo_mixed_batch.argtypes = [P, P, P, P, P, P, U64]
        lib.dyo_resize.argtypes = [P, I32, I32]
        lib.dyo_resize.restype = I32
        lib.dyo_stats.argtypes = [P, C.POINTER(_Stats)]
        lib.dyo_dump.argtypes = [P, P, P, P, U64]
        lib.dyo_dump.restype = U64
        lib.dyo_check_invariants.argtypes = [P, C.c_char_p, U64]
        lib.dyo_check_invariants.restype = U64
        lib.dyo_hash_x.argtypes = [P, U32, U32]
        lib.dyo_hash_x.restype = U64
        lib.dyo_pair.argtypes = [P, U32, C.POINTER(U32), C.POINTER(U32)]
        lib.dyo_bucket.argtypes = [P, U32, U32]
        lib.dyo_bucket.restype = U64
        lib.dyo_hash_params.argtypes = [P, P, P]
        lib.dyo_check_layout.argtypes = [P, P, P, P, P, U64]
        lib.dyo_check_layout.restype = U64
        lib.dyo_poke.argtypes = [P, U32, U64, U32, U32, U32]
        lib.dyo_poke.restype = I32
        lib.dyo_peek.argtypes = [P, U32, U64, U32]
        lib.dyo_peek.restype = U64
        lib.dyo_debug_adjust_count.argtypes = [P, U32, C.c_int64]
        lib.dyo_debug_adjust_count.restype = I32
        lib.dyo_place_one.argtypes = [P, U32, U32]
        lib.dyo_place_one.restype = I32
        _lib = lib
    return _lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


class OracleTable:
    """Sequential DyCuckoo (oracle/dyc_oracle.c)."""

    def __init__(self, d: int = 4, init_capacity: int = 4096, alpha: float = 0.3,
                 beta: float = 0.85, bucket_slots: int = 4, seed: int = 0x5EED0001,
                 max_hops: int = 64, policy: int = FIRST_FIT):
        self._lib = oracle_lib()
        self.d, self.B = d, bucket_slots
        self._t = self._lib.dyo_create(d, bucket_slots, init_capacity, alpha, beta, seed,
                                       max_hops, policy)
        if not self._t:
            raise ValueError("dyo_create rejected the arguments")

    def close(self):
        if self._t:
            self._lib.dyo_destroy(self._t)
            self._t = None

    __del__ = close

    # -- batches -------------------------------------------------------------
    def insert(self, keys: np.ndarray, values: np.ndarray) -> np.ndarray:
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        values = np.ascontiguousarray(values, dtype=np.uint32)
        st = np.zeros(keys.size, dtype=np.uint8)
        self._lib.dyo_insert_batch(self._t, _ptr(keys), _ptr(values), _ptr(st), keys.size)
        return st

    def find(self, keys: np.ndarray) -> Tuple[np.ndarray, np.ndarray]:
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        v = np.zeros(keys.size, dtype=np.uint32)
        f = np.zeros(keys.size, dtype=np.uint8)
        self._lib.dyo_find_batch(self._t, _ptr(keys), _ptr(v), _ptr(f), keys.size)
        return v, f

    def delete(self, keys: np.ndarray) -> Tuple[np.ndarray, np.ndarray]:
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        v = np.zeros(keys.size, dtype=np.uint32)
        st = np.zeros(keys.size, dtype=np.uint8)
        self._lib.dyo_delete_batch(self._t, _ptr(keys), _ptr(v), _ptr(st), keys.size)
        return v, st

    def mixed(self, ops: np.ndarray, keys: np.ndarray, values: np.ndarray):
        ops = np.ascontiguousarray(ops, dtype=np.uint8)
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        values = np.ascontiguousarray(values, dtype=np.uint32)
        v = np.zeros(keys.size, dtype=np.uint32)
        st = np.zeros(keys.size, dtype=np.uint8)
        self._lib.dyo_mixed_batch(self._t, _ptr(ops), _ptr(keys), _ptr(values), _ptr(v), _ptr(st), keys.size)
        return v, st

    def resize(self, direction: int, subtable: int = -1) -> int:
        return int(self._lib.dyo_resize(self._t, direction, subtable))

    # -- inspection ----------------------------------------------------------
    def stats(self) -> Dict:
        s = _Stats()
        self._lib.dyo_stats(self._t, C.byref(s))
        d = s.d
        return dict(m=s.m, N=s.N, d=d, B=s.B, buckets=list(s.buckets[:d]),
                    count=list(s.count[:d]), n_upsize=s.n_upsize, n_downsize=s.n_downsize,
                    n_fail_upsize=s.n_fail_upsize, n_residual=s.n_residual,
                    n_evict=s.n_evict, max_probes=s.max_probes,
                    n_second_table=s.n_second_table, invariant_errors=s.invariant_errors,
                    fill=(s.m / s.N) if s.N else 0.0)

    def dump(self):
        n = int(self._lib.dyo_dump(self._t, None, None, None, 0))
        kv = np.zeros(n, dtype=np.uint64)
        tb = np.zeros(n, dtype=np.uint32)
        bk = np.zeros(n, dtype=np.uint64)
        self._lib.dyo_dump(self._t, _ptr(kv), _ptr(tb), _ptr(bk), n)
        return kv, tb, bk

    def contents(self) -> Dict[int, int]:
        kv, _, _ = self.dump()
        return {int(x & 0xFFFFFFFF): int(x >> 32) for x in kv}

    def sorted_kv(self) -> np.ndarray:
        kv, _, _ = self.dump()
        keys = (kv & np.uint64(0xFFFFFFFF)).astype(np.uint32)
        return kv[np.argsort(keys, kind="stable")]

    def check_invariants(self) -> Tuple[int, str]:
        buf = C.create_string_buffer(256)
        bad = int(self._lib.dyo_check_invariants(self._t, buf, 256))
        return bad, buf.value.decode()

    def check_layout(self, buckets, keys, tables, bucket_idx) -> int:
        nb = np.ascontiguousarray(buckets, dtype=np.uint64)
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        tables = np.ascontiguousarray(tables, dtype=np.uint32)
        bucket_idx = np.ascontiguousarray(bucket_idx, dtype=np.uint64)
        return int(self._lib.dyo_check_layout(self._t, _ptr(nb), _ptr(keys), _ptr(tables),
                                              _ptr(bucket_idx), keys.size))

    # -- hash spec exposure (test vectors) -------------------------------------
    def hash_x(self, s: int, k: int) -> int:
        return int(self._lib.dyo_hash_x(self._t, s, k))

    def pair(self, k: int) -> Tuple[int, int]:
        a, b = C.c_uint32(), C.c_uint32()
        self._lib.dyo_pair(self._t, k, C.byref(a), C.byref(b))
        return a.value, b.value

    def bucket(self, t: int, k: int) -> int:
        return int(self._lib.dyo_bucket(self._t, t, k))

    def hash_params(self) -> Tuple[np.ndarray, np.ndarray]:
        a = np.zeros(self.d + 2, dtype=np.uint64)
        b = np.zeros(self.d + 2, dtype=np.uint64)
        self._lib.dyo_hash_params(self._t, _ptr(a), _ptr(b))
        return a, b

    # -- scripted-scenario hooks ------------------------------------------------
    def poke(self, t: int, b: int, s: int, key: int, val: int) -> None:
        if self._lib.dyo_poke(self._t, t, b, s, key, val) != 0:
            raise IndexError("poke out of range")

    def peek(self, t: int, b: int, s: int) -> Tuple[int, int]:
        x = int(self._lib.dyo_peek(self._t, t, b, s))
        return x & 0xFFFFFFFF, x >> 32

    def debug_adjust_count(self, t: int, delta: int) -> None:
        """Corrupts the counter m_t (negative pins of check_invariants, I4)."""
        if self._lib.dyo_debug_adjust_count(self._t, t, delta) != 0:
            raise IndexError("subtable out of range")

    def place_one(self, key: int, val: int) -> int:
        return int(self._lib.dyo_place_one(self._t, key, val))
