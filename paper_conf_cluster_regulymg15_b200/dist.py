"""Multi-process plumbing for one-process-per-GPU runs (torch.distributed):
chunk-grid choice, NCCL unique-id broadcast and max-over-ranks timing.
The halo exchange and the dt MIN all-reduce themselves run inside
libclover.so over NCCL; this module only sets them up.  GlooHostTransport
carries the same three collectives over a gloo process group on host
buffers (clover_host_transport): ranks without NCCL, e.g. several processes
sharing one GPU, which NCCL refuses.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def chunk_grid(nranks: int, nx: int, ny: int, strips: bool = True) -> tuple[int, int]:
    """px x py chunks for nranks ranks, one chunk per rank.  Default: y
    strips (px = 1) while each strip keeps >= 16 rows, so every chunk has
    both x walls and the fused x-sweep kernel applies;
    otherwise, or with strips=False, the most square chunks, splitting the
    longer axis first (the reference's clover_decompose idea; SURVEY 8(e):
    2 -> 1x2 on a square mesh)."""
    if strips and ny // nranks >= 16:
        return 1, nranks
    best = None
    for px in range(1, nranks + 1):
        if nranks % px:
            continue
        py = nranks // px
        lx, ly = nx / px, ny / py
        score = (max(lx, ly) / min(lx, ly), -py)  # squarest, then prefer y splits
        if best is None or score < best[0]:
            best = (score, px, py)
    return best[1], best[2]


def weak_mesh(nranks: int, per: int = 3840) -> tuple[int, int, int, int]:
    """Reading A4: per^2 cells per rank on the fixed [0,10]^2
    domain, the global mesh growing in both axes -- 1: per^2, 2: 2per x per,
    4: (2per)^2, 8: 4per x 2per (nranks = a*b, b the largest power of two
    with b*b <= nranks, a = nranks/b); y strips (1 x nranks chunk grid), so
    every rank owns per^2 cells and both sweeps stay fused."""
    b = 1
    while (2 * b) * (2 * b) <= nranks and nranks % (2 * b) == 0:
        b *= 2
    a = nranks // b
    return per * a, per * b, 1, nranks


def share_unique_id(make_id) -> bytes:
    """Rank 0 creates the 128-byte NCCL unique id (make_id()), every rank
    returns the same bytes."""
    obj = [make_id() if dist.get_rank() == 0 else None]
    dist.broadcast_object_list(obj, src=0)
    uid = obj[0]
    if not isinstance(uid, (bytes, bytearray)) or len(uid) != 128:
        raise ValueError("bad NCCL unique id")
    return bytes(uid)


def max_over_ranks(value: float, device=None) -> float:
    """Max of a per-rank timing over all ranks (the bench reports the
    slowest rank)."""
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


class GlooHostTransport:
    """clover_host_transport over torch.distributed (gloo, CPU tensors).
    The library hands host buffers; these callbacks only move them (halo
    messages point to point, the dt bit pattern MIN, summary/readback
    all-gather) -- no arithmetic of the method."""

    def __init__(self, group=None):
        self.group = group

    def _sendrecv(self, user, n, peer, send, nsend, recv, nrecv):
        import numpy as np
        try:
            reqs = []
            for i in range(n):
                a = np.ctypeslib.as_array(send[i], shape=(int(nsend[i]),))
                reqs.append(dist.isend(torch.from_numpy(a), int(peer[i]), group=self.group))
            for i in range(n):
                b = np.ctypeslib.as_array(recv[i], shape=(int(nrecv[i]),))
                reqs.append(dist.irecv(torch.from_numpy(b), int(peer[i]), group=self.group))
            for r in reqs:
                r.wait()
            return 0
        except Exception:  # noqa: BLE001 -- reported to the library as a failed call
            return 1

    def _allreduce(self, user, value):
        try:
            # positive doubles' bit patterns fit int64 and order like the values
            t = torch.tensor([int(value[0])], dtype=torch.int64)
            dist.all_reduce(t, op=dist.ReduceOp.MIN, group=self.group)
            value[0] = int(t.item())
            return 0
        except Exception:  # noqa: BLE001
            return 1

    def _allgather(self, user, send, count, recv):
        import numpy as np
        try:
            world = dist.get_world_size(self.group)
            a = torch.from_numpy(np.ctypeslib.as_array(send, shape=(int(count),)).copy())
            outs = [torch.empty(int(count), dtype=torch.float64) for _ in range(world)]
            dist.all_gather(outs, a, group=self.group)
            r = np.ctypeslib.as_array(recv, shape=(world * int(count),))
            for i, o in enumerate(outs):
                r[i * int(count):(i + 1) * int(count)] = o.numpy()
            return 0
        except Exception:  # noqa: BLE001
            return 1

    def c_struct(self):
        from .clover import (ALLGATHER_FN, ALLREDUCE_FN, SENDRECV_FN, CloverHostTransport)
        self._cb = (SENDRECV_FN(self._sendrecv), ALLREDUCE_FN(self._allreduce),
                    ALLGATHER_FN(self._allgather))
        return CloverHostTransport(None, *self._cb)
