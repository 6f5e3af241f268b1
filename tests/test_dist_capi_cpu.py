"""world_size-2 gloo test of the sharded C ABI's host side (dyc_dist_*): the
NCCL unique id is created by rank 0 through dyc_dist_get_unique_id and
broadcast over torch.distributed (the only thing torch.distributed does for
the sharded path), every rank ends up with the same 128 bytes, and
dyc_dist_create_ex validates its arguments and fails loudly (no CPU fallback)
when there is no device.  The batch calls themselves need a GPU:
tests/test_gpu_sharded.py.  No GPU needed here."""
import ctypes as C
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icde_lizlhs21_b200 import _lib as L
    from paper_conf_icde_lizlhs21_b200.sharded import ShardedTable, broadcast_unique_id
    out = {}
    uid = broadcast_unique_id()
    ids = [None] * world
    dist.all_gather_object(ids, uid)
    out["same_id"] = all(i == ids[0] for i in ids) and len(ids[0]) == 128 and any(ids[0])
    lib = L.load_library()
    cfg = L.dyc_config()
    lib.dyc_config_default(C.byref(cfg))
    h = C.c_void_p()
    buf = C.create_string_buffer(uid, 128)
    out["bad_rank"] = lib.dyc_dist_create_ex(C.byref(cfg), buf, world, world, 1, C.byref(h)) == L.DYC_ERR_INVALID_ARG
    out["no_id"] = lib.dyc_dist_create_ex(C.byref(cfg), None, rank, world, 1, C.byref(h)) == L.DYC_ERR_INVALID_ARG
    out["no_shards"] = lib.dyc_dist_create_ex(C.byref(cfg), buf, rank, world, 0, C.byref(h)) == L.DYC_ERR_INVALID_ARG
    out["too_many"] = lib.dyc_dist_create_ex(C.byref(cfg), buf, rank, world, 1000, C.byref(h)) == L.DYC_ERR_INVALID_ARG
    cfg.alpha = 0.9
    out["bad_cfg"] = lib.dyc_dist_create_ex(C.byref(cfg), buf, rank, world, 1, C.byref(h)) in (
        L.DYC_ERR_INVALID_ARG, L.DYC_ERR_NO_DEVICE)
    if not torch.cuda.is_available():
        try:
            ShardedTable(d=4, init_capacity=1 << 12, rank=rank, world=world, unique_id=uid)
            out["no_device"] = False
        except L.DycError as e:
            out["no_device"] = e.code == L.DYC_ERR_NO_DEVICE
    q.put((rank, out))
    dist.destroy_process_group()


def test_unique_id_broadcast_and_create_checks_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert all(res[r].values()), res[r]


def test_unique_id_without_gpu():
    from paper_conf_icde_lizlhs21_b200.sharded import new_unique_id
    a, b = new_unique_id(), new_unique_id()
    assert len(a) == len(b) == 128 and a != b


def test_world_one_needs_no_id():
    """broadcast_unique_id returns None outside a process group / with one rank."""
    from paper_conf_icde_lizlhs21_b200.sharded import broadcast_unique_id
    if dist.is_initialized():
        pytest.skip("a process group is already initialised")
    assert broadcast_unique_id() is None
