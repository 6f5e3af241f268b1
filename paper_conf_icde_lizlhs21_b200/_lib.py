"""ctypes binding of libdyc.so (include/dycuckoo.h): argument marshalling only.

Every function of the C ABI is exposed under its C name with the same argument
order; pointers are passed as Python ints (device addresses, e.g.
``tensor.data_ptr()``) and streams as ints (``torch.cuda.Stream.cuda_stream``).
There is no CPU fallback: loading fails loudly when the library is missing.
"""
from __future__ import annotations

import ctypes as C
import os

from .build import LIB

DYC_MAX_D = 16
DYC_EMPTY_KEY = 0xFFFFFFFF
DYC_NOT_FOUND = 0xFFFFFFFF

DYC_OK, DYC_ERR_INVALID_ARG, DYC_ERR_OOM, DYC_ERR_CUDA, DYC_ERR_INSERT_FAILED, DYC_ERR_NO_DEVICE, DYC_ERR_NCCL = range(7)
DYC_NCCL_UNIQUE_ID_BYTES = 128
DYC_PLACE_PAPER_WEIGHTED = 1
DYC_RESIZE_IN_PLACE = 2
DYC_STAGED_OFF = 4
DYC_STAGED_FORCE = 8
DYC_RESIZE_SPLIT, DYC_RESIZE_REINSERT_SUBTABLE, DYC_RESIZE_REHASH_ALL = range(3)
DYC_PROF_KINDS = 16
DYC_GATHER_WRITE, DYC_GATHER_CAS, DYC_GATHER_SECTOR = 1, 2, 4
PROF_NAMES = ["k_find", "k_upsert", "k_place", "k_delete", "k_upsize", "k_downsize", "k_reinsert", "other",
              "st_hist", "st_scatter", "st_apply", "st_unperm"]
_STATUS_NAMES = ["DYC_OK", "DYC_ERR_INVALID_ARG", "DYC_ERR_OOM", "DYC_ERR_CUDA",
                 "DYC_ERR_INSERT_FAILED", "DYC_ERR_NO_DEVICE", "DYC_ERR_NCCL"]


class dyc_config(C.Structure):
    _fields_ = [("d", C.c_uint32), ("bucket_slots", C.c_uint32), ("alpha", C.c_double),
                ("beta", C.c_double), ("init_capacity", C.c_uint64), ("seed", C.c_uint64),
                ("max_hops", C.c_uint32), ("flags", C.c_uint32)]


class dyc_stats_t(C.Structure):
    _fields_ = [("m", C.c_uint64), ("N", C.c_uint64), ("d", C.c_uint32), ("B", C.c_uint32),
                ("buckets", C.c_uint64 * DYC_MAX_D), ("count", C.c_uint64 * DYC_MAX_D),
                ("fill", C.c_double), ("n_upsize", C.c_uint64), ("n_downsize", C.c_uint64),
                ("n_fail_upsize", C.c_uint64), ("n_residual", C.c_uint64), ("n_evict", C.c_uint64),
                ("n_place_retry", C.c_uint64), ("n_second_table", C.c_uint64),
                ("bytes_allocated", C.c_uint64), ("last_insert_new", C.c_uint64),
                ("last_insert_pending", C.c_uint64), ("last_insert_evictions", C.c_uint64),
                ("bytes_cached", C.c_uint64), ("n_live_resize", C.c_uint64), ("n_deferred", C.c_uint64),
                ("n_device_alloc", C.c_uint64), ("alloc_ms", C.c_double),
                ("n_sync", C.c_uint64), ("sync_ms", C.c_double), ("n_pending", C.c_uint64),
                ("vm_subtables", C.c_uint64), ("vm_mapped_bytes", C.c_uint64), ("n_vm_map", C.c_uint64),
                ("n_vm_unmap", C.c_uint64), ("n_staged", C.c_uint64)]


class dyw_config(C.Structure):
    _fields_ = [("d", C.c_uint32), ("value_words", C.c_uint32), ("mode", C.c_uint32), ("max_hops", C.c_uint32),
                ("alpha", C.c_double), ("beta", C.c_double), ("init_capacity", C.c_uint64), ("seed", C.c_uint64)]


class dyw_stats_t(C.Structure):
    _fields_ = [("m", C.c_uint64), ("N", C.c_uint64), ("d", C.c_uint32), ("B", C.c_uint32),
                ("W", C.c_uint32), ("mode", C.c_uint32),
                ("buckets", C.c_uint64 * DYC_MAX_D), ("count", C.c_uint64 * DYC_MAX_D),
                ("fill", C.c_double), ("n_upsize", C.c_uint64), ("n_downsize", C.c_uint64),
                ("n_fail_upsize", C.c_uint64), ("n_residual", C.c_uint64), ("n_evict", C.c_uint64),
                ("n_lock_fail", C.c_uint64), ("last_insert_new", C.c_uint64),
                ("last_insert_pending", C.c_uint64), ("bytes_allocated", C.c_uint64)]


DYW_MODE_VOTER, DYW_MODE_GROUPED, DYW_MODE_LOCKFREE = 0, 1, 2


class DycError(RuntimeError):
    def __init__(self, code: int, fn: str, msg: str):
        name = _STATUS_NAMES[code] if 0 <= code < len(_STATUS_NAMES) else str(code)
        super().__init__(f"{fn} -> {name}: {msg}")
        self.code = code


_P, _U8, _U32, _U64, _I, _D = C.c_void_p, C.c_uint8, C.c_uint32, C.c_uint64, C.c_int, C.c_double
_TP = C.c_void_p   # dyc_table*

# name -> (restype, argtypes)
SIGNATURES = {
    "dyc_config_default": (_I, [C.POINTER(dyc_config)]),
    "dyc_create": (_I, [_U32, _U64, _D, _D, C.POINTER(_TP)]),
    "dyc_create_ex": (_I, [C.POINTER(dyc_config), C.POINTER(_TP)]),
    "dyc_destroy": (_I, [_TP]),
    "dyc_insert_batch": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_find_batch": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_insert_begin": (_I, [_TP, _U64, _P]),
    "dyc_insert_part": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_insert_end": (_I, [_TP, _P]),
    "dyc_delete_begin": (_I, [_TP, _U64, _P]),
    "dyc_delete_part": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_delete_end": (_I, [_TP, _P]),
    "dyc_delete_batch": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_mixed_batch": (_I, [_TP, _P, _P, _P, _P, _P, _U64, _P]),
    "dyc_resize": (_I, [_TP, _I, _I, _P]),
    "dyc_resize_ex": (_I, [_TP, _I, _I, _I, _P]),
    "dyc_resize_begin": (_I, [_TP, _I, _I, _P, _P]),
    # wide-key table (include/dycuckoo_wide.h, NEXT-3)
    "dyw_config_default": (_I, [C.POINTER(dyw_config)]),
    "dyw_create": (_I, [C.POINTER(dyw_config), C.POINTER(_TP)]),
    "dyw_destroy": (_I, [_TP]),
    "dyw_insert_batch": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyw_find_batch": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyw_delete_batch": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyw_resize": (_I, [_TP, _I, _I, _P]),
    "dyw_clear": (_I, [_TP, _P]),
    "dyw_stats": (_I, [_TP, C.POINTER(dyw_stats_t), _P]),
    "dyw_dump": (_I, [_TP, _P, _P, _P, _P, _U64, C.POINTER(_U64), _P]),
    "dyw_hash_probe": (_I, [_TP, _P, _U64, _P, _P, _P]),
    "dyw_launch_count": (_U64, [_TP, _I]),
    "dyc_resize_commit": (_I, [_TP, _P]),
    "dyc_resize_query": (_I, [_TP, C.POINTER(_I), C.POINTER(_I)]),
    "dyc_clear": (_I, [_TP, _P]),
    "dyc_trim": (_I, [_TP]),
    "dyc_stats": (_I, [_TP, C.POINTER(dyc_stats_t), _P]),
    "dyc_dump": (_I, [_TP, _P, _P, _P, _U64, C.POINTER(_U64), _P]),
    "dyc_shape": (_I, [_TP, _P, C.POINTER(_U64), C.POINTER(_U64), C.POINTER(_U64)]),
    "dyc_hash_params": (_I, [_TP, _P, _P]),
    "dyc_hash_probe": (_I, [_TP, _P, _U64, _P, _P, _P]),
    "dyc_insert_batch_host": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_find_batch_host": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_delete_batch_host": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_launch_count": (_U64, [_TP, _I]),
    "dyc_profile_enable": (_I, [_TP, _I]),
    "dyc_profile_read": (_I, [_TP, _P, _P]),
    "dyc_probe_count_enable": (_I, [_TP, _I]),
    "dyc_probe_count_read": (_I, [_TP, _P]),
    "dyc_clean_mask": (_I, [_TP, C.POINTER(_U32)]),
    "dyc_route_count": (_I, [_TP, _P, _U64, _U32, _P, _P]),
    "dyc_route_scatter": (_I, [_TP, _P, _P, _P, _U64, _U32, _P, _P, _P, _P, _P, _P, _P]),
    "dyc_route_unpermute": (_I, [_P, _U64, _P, _P, _P, _P, _P]),
    "dyc_ipc_alloc": (_I, [_U64, C.POINTER(C.c_void_p)]),
    "dyc_ipc_free": (_I, [_P]),
    "dyc_ipc_get_handle": (_I, [_P, _P]),
    "dyc_ipc_open": (_I, [_P, C.POINTER(C.c_void_p)]),
    "dyc_ipc_close": (_I, [_P]),
    "dyc_route_push": (_I, [_TP, _P, _P, _P, _U64, _U32, _U32, _P, _P, _U64, _P]),
    "dyc_route_reply": (_I, [_P, _U64, _U64, _P, _P, _U32, _P, _P, _P]),
    "dyc_bench_gather": (_I, [_P, _U64, _U64, _U32, _U64, _P, _P]),
    "dyc_bench_gather_ex": (_I, [_P, _U64, _U64, _U32, _U64, _U32, _P, _P]),
    "dyc_set_l2_fetch_granularity": (_I, [_U32]),
    "dyc_get_l2_fetch_granularity": (_I, [C.POINTER(_U32)]),
    # sharded table (dyc_dist_*, NCCL between processes, local virtual shards)
    "dyc_dist_get_unique_id": (_I, [_P]),
    "dyc_dist_create": (_I, [_U32, _U64, _D, _D, _P, _I, _I, C.POINTER(_TP)]),
    "dyc_dist_create_ex": (_I, [C.POINTER(dyc_config), _P, _I, _I, _U32, C.POINTER(_TP)]),
    "dyc_dist_destroy": (_I, [_TP]),
    "dyc_dist_insert_batch": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_dist_find_batch": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_dist_delete_batch": (_I, [_TP, _P, _P, _P, _U64, _P]),
    "dyc_dist_mixed_batch": (_I, [_TP, _P, _P, _P, _P, _P, _U64, _P]),
    "dyc_dist_info": (_I, [_TP, C.POINTER(_I), C.POINTER(_I), C.POINTER(_U32), C.POINTER(_U64)]),
    "dyc_dist_shard": (_I, [_TP, _U32, C.POINTER(_TP)]),
    "dyc_last_error": (C.c_char_p, []),
    "dyc_version": (C.c_char_p, []),
}

_lib = None


def load_library(path: str = None):
    """Loads libdyc.so (building it first if nvcc is present and it is stale).
    DYC_LIB overrides the path (tuning experiments only)."""
    global _lib
    if _lib is not None:
        return _lib
    path = path or os.environ.get("DYC_LIB") or LIB
    if not os.path.exists(path):
        try:
            from .build import build_library
            build_library()
        except Exception as e:  # noqa: BLE001
            raise RuntimeError(f"libdyc.so is missing and could not be built: {e}") from e
    lib = C.CDLL(path)
    for name, (res, args) in SIGNATURES.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    _lib = lib
    return lib


def last_error() -> str:
    return load_library().dyc_last_error().decode(errors="replace")


def check(code: int, fn: str) -> None:
    if code != DYC_OK:
        raise DycError(code, fn, last_error())


def _wrap(name):
    def f(*args):
        return getattr(load_library(), name)(*args)
    f.__name__ = name
    f.__doc__ = f"C ABI function {name} (include/dycuckoo.h)."
    return f


# module-level functions with the C names
for _n in SIGNATURES:
    globals()[_n] = _wrap(_n)
