"""ctypes wrapper of oracle/brute_map.cpp (std::unordered_map brute force):
TEST INFRASTRUCTURE and CPU BASELINE (ii) only."""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "brute_map.cpp")
_LIB = os.path.join(_HERE, "libbrute_map.so")


def build_brute(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-Wall", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def brute_lib():
    global _lib
    if _lib is None:
        lib = C.CDLL(build_brute())
        P, U64 = C.c_void_p, C.c_uint64
        lib.bm_create.restype = P
        lib.bm_create.argtypes = [U64]
        lib.bm_destroy.argtypes = [P]
        lib.bm_size.restype = U64
        lib.bm_size.argtypes = [P]
        for name in ("bm_insert_batch", "bm_find_batch", "bm_delete_batch"):
            getattr(lib, name).argtypes = [P, P, P, P, U64]
        lib.bm_mixed_batch.argtypes = [P, P, P, P, P, P, U64]
        _lib = lib
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


class BruteMapCpp:
    def __init__(self, reserve: int = 0):
        self._lib = brute_lib()
        self._h = self._lib.bm_create(reserve)

    def close(self):
        if self._h:
            self._lib.bm_destroy(self._h)
            self._h = None

    __del__ = close

    def __len__(self):
        return int(self._lib.bm_size(self._h))

    def insert(self, keys, vals):
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        vals = np.ascontiguousarray(vals, dtype=np.uint32)
        st = np.zeros(keys.size, dtype=np.uint8)
        self._lib.bm_insert_batch(self._h, _p(keys), _p(vals), _p(st), keys.size)
        return st

    def find(self, keys):
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        v = np.zeros(keys.size, dtype=np.uint32)
        f = np.zeros(keys.size, dtype=np.uint8)
        self._lib.bm_find_batch(self._h, _p(keys), _p(v), _p(f), keys.size)
        return v, f

    def delete(self, keys):
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        v = np.zeros(keys.size, dtype=np.uint32)
        st = np.zeros(keys.size, dtype=np.uint8)
        self._lib.bm_delete_batch(self._h, _p(keys), _p(v), _p(st), keys.size)
        return v, st

    def mixed(self, ops, keys, vals):
        ops = np.ascontiguousarray(ops, dtype=np.uint8)
        keys = np.ascontiguousarray(keys, dtype=np.uint32)
        vals = np.ascontiguousarray(vals, dtype=np.uint32)
        v = np.zeros(keys.size, dtype=np.uint32)
        st = np.zeros(keys.size, dtype=np.uint8)
        self._lib.bm_mixed_batch(self._h, _p(ops), _p(keys), _p(vals), _p(v), _p(st), keys.size)
        return v, st
