"""Multi-process host logic on CPU: world_size 2 over gloo (the N>1 path of
bench.py minus the GPUs): unique-id broadcast, max-over-ranks timing, chunk
grids and per-rank workspace sizing through the C ABI."""
from __future__ import annotations

import ctypes
import os
import socket

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_cluster_regulymg15_b200 import dist as cdist


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
    try:
        uid = cdist.share_unique_id(lambda: bytes(range(128)))
        t = cdist.max_over_ranks(1.5 + rank)
        from paper_conf_cluster_regulymg15_b200 import clover as cb
        from workloads import bm_deck
        nx, ny, px, py = cdist.weak_mesh(world, per=64)
        g = cb.grid_from_deck(bm_deck(nx, ny))
        buf = ctypes.create_string_buffer(uid, 128)
        d = cb.CloverDist(rank=rank, nranks=world, px=px, py=py,
                          nccl_unique_id=ctypes.cast(buf, ctypes.c_void_p))
        nb = ctypes.c_int64()
        rc = cb.load().clover_workspace_bytes(ctypes.byref(g), ctypes.byref(d), ctypes.byref(nb))
        sizes = [None] * world
        dist.all_gather_object(sizes, (rc, nb.value))
        q.put((rank, uid, t, sizes, (nx, ny, px, py)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_two_ranks_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    assert all(r[1] == bytes(range(128)) for r in res)
    assert all(r[2] == 1.5 + world - 1 for r in res)
    sizes = res[0][3]
    assert all(rc == 0 for rc, _ in sizes)
    assert sizes[0][1] == sizes[1][1] > 0  # equal chunks -> equal workspaces
    assert res[0][4] == (128, 64, 1, 2)


def test_chunk_grid_and_weak_series():
    assert cdist.chunk_grid(1, 100, 100) == (1, 1)
    assert cdist.chunk_grid(2, 7680, 7680) == (1, 2)
    assert cdist.chunk_grid(8, 7680, 7680) == (1, 8)
    assert cdist.chunk_grid(4, 7680, 7680, strips=False) == (2, 2)
    assert cdist.chunk_grid(8, 7680, 7680, strips=False) in ((2, 4), (4, 2))
    assert cdist.chunk_grid(2, 1000, 100, strips=False) == (2, 1)
    assert cdist.chunk_grid(8, 100, 64)[0] > 1  # strips would be < 16 rows
    # SURVEY reading A4: per-GPU 3840^2 on [0,10]^2: 1: 3840^2, 2: 7680x3840,
    # 4: 7680^2, 8: 15360x7680, y strips
    assert cdist.weak_mesh(1) == (3840, 3840, 1, 1)
    assert cdist.weak_mesh(2) == (7680, 3840, 1, 2)
    assert cdist.weak_mesh(4) == (7680, 7680, 1, 4)
    assert cdist.weak_mesh(8) == (15360, 7680, 1, 8)
    for n in (1, 2, 4, 8, 3, 6):
        nx, ny, px, py = cdist.weak_mesh(n)
        assert nx * ny == n * 3840 * 3840 and px * py == n
