"""Multi-rank path of the library with real processes: two or
four processes, each one rank owning one chunk, all on the one GPU of the
box, exchanging halos, the dt MIN and the summary/readback gathers through
the host transport over gloo (clover_host_transport; NCCL refuses two ranks
on one device).  Everything above the transport -- rank-to-chunk mapping,
message packing and matching, the dt reduction, the deterministic summary,
the cross-rank field gather -- is the production multi-rank code.

Bar: every state field, the dt history and the summary bit-identical to the
same deck on one chunk, and the fields bitwise equal to the oracle.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

from oracle import Oracle
from workloads import fuzz_deck, point_deck

pytestmark = pytest.mark.gpu

STATE = ("density0", "energy0", "xvel0", "yvel0")


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, deck, px, py, steps, out, deep=False):
    import torch
    import torch.distributed as dist

    from paper_conf_cluster_regulymg15_b200 import Clover
    from paper_conf_cluster_regulymg15_b200.dist import GlooHostTransport

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    sim = Clover(deck, px=px, py=py, rank=rank, nranks=world, host_transport=GlooHostTransport())
    sim.set_deep_halo(deep)  # (on by default: the plain cases keep the per-phase schedule)
    assert sim.deep_halo_active() == deep
    sim.step(steps)
    fields = {f: sim.read(f) for f in STATE}
    summ = sim.field_summary()
    dts = sim.dt_history(1, steps)
    clock = sim.clock()
    if rank == 0:
        np.savez(out, dts=dts, **fields,
                 summ=np.array([summ[k] for k in ("vol", "mass", "ie", "ke", "press")]),
                 clock=np.array([clock["step"], clock["time"]]))
    sim.close()
    dist.barrier()
    dist.destroy_process_group()


def _run(world, deck, px, py, steps, tmp_path, deep=False):
    import torch.multiprocessing as mp
    out = str(tmp_path / f"r0_{world}_{px}x{py}_{int(deep)}.npz")
    ctx = mp.start_processes(_worker, args=(world, _free_port(), deck, px, py, steps, out, deep),
                             nprocs=world, join=False, start_method="spawn")
    while not ctx.join(timeout=240):
        pass
    return np.load(out)


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


@pytest.mark.timeout(600)
@pytest.mark.parametrize("world,px,py,deck,deep", [
    (2, 1, 2, "fuzz", False),  # y strips: the launcher's default decomposition
    (2, 2, 1, "point", False),  # x strips: separate x kernels, fused y
    (4, 2, 2, "fuzz", False),  # four ranks, 4-rank corners
    (2, 1, 2, "fuzz", True),   # deep halos: one 7-row state exchange per step
    (4, 1, 4, "point", True),  # deep halos, 16-row strips (the minimum)
])
def test_processes_match_one_chunk_and_oracle(torch_cuda, tmp_path, world, px, py, deck, deep):
    from paper_conf_cluster_regulymg15_b200 import Clover
    d = fuzz_deck(21, nx=72, ny=64) if deck == "fuzz" else point_deck(72, 64)
    steps = 12
    got = _run(world, d, px, py, steps, tmp_path, deep)
    one = Clover(d)
    one.step(steps)
    o = Oracle(d)
    dts = o.step(steps)
    assert np.array_equal(got["dts"], one.dt_history(1, steps))
    assert np.array_equal(got["dts"], dts)
    for f in STATE:
        assert np.array_equal(got[f], one.read(f)), f
        assert np.array_equal(got[f], o.read(f)), f
    s1 = one.field_summary()
    assert np.array_equal(got["summ"], np.array([s1[k] for k in ("vol", "mass", "ie", "ke", "press")]))
    assert got["clock"][0] == steps and got["clock"][1] == one.clock()["time"]
    one.close()
