"""Cost of the halo-exchange machinery on one GPU: the same bm mesh as one
chunk and as px x py local chunks (device-to-device exchange phases), with
the fused y sweep across y chunk boundaries (default) or only at walls
(round-1 schedule: separate y kernels + an extra exchange phase), and
through the virtual-remote packing path (pack -> staging -> unpack, the
multi-GPU message layout), by device copy and through a one-rank NCCL
communicator, and as device-initiated stores into a one-rank NCCL symmetric
window (virtual_lsa*); each also with deep halos (one 7-row state exchange
per step, *_deep).  Prints one JSON line.
usage: chunk_overhead.py NX NY PX PY [STEPS]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_regulymg15_b200 import Clover  # noqa: E402
from workloads import bm_deck  # noqa: E402

nx, ny, px, py = (int(a) for a in sys.argv[1:5])
steps = int(sys.argv[5]) if len(sys.argv) > 5 else 20
torch.cuda.set_device(0)
deck = bm_deck(nx, ny, end_step=steps, ymax=10.0 * ny / nx)
# (square cells: the domain grows with the mesh)


def run(p, q, vr=0, walls_only=False, overlap=False, deep=False):
    sim = Clover(deck, px=p, py=q)
    sim.set_deep_halo(deep)
    if walls_only:
        sim.debug_set_fusion(True, walls_only=True)
    if vr:
        sim.debug_set_virtual_remote(True, nccl=vr == 2, lsa=vr == 3)
    sim.debug_set_overlap(overlap)
    sim.step(3)
    sim.sync()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(sim.stream)
    sim.step(steps)
    e1.record(sim.stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    kps = sim.kernels_per_step()
    sim.close()
    return ms, kps


one, k1 = run(1, 1)
res = {"mesh": [nx, ny], "chunks": [px, py], "steps": steps, "one_chunk_ms": one, "one_chunk_kernels": k1}
# one rank's share alone: a single chunk of the per-rank size (walls on all
# sides, same cell size) -- what a rank of a real px*py run computes per
# step minus the exchange; nchunks x this = the serialised one-GPU ideal
cx, cy = nx // px, ny // py
deck_full = deck
deck = bm_deck(cx, cy, end_step=steps, xmax=10.0 * cx / nx, ymax=10.0 * cy / ny)
alone, _ = run(1, 1)
deck = deck_full
res["rank_chunk"] = [cx, cy]
res["rank_chunk_alone_ms"] = alone
res["serial_ideal_ms"] = alone * px * py
res["strong_scaling_efficiency_bound"] = one / (px * py * alone)
for name, kw in (("local_fused", {}), ("local_walls_only", dict(walls_only=True)),
                 ("virtual_remote", dict(vr=1)), ("virtual_nccl", dict(vr=2)),
                 ("virtual_remote_overlap", dict(vr=1, overlap=True)),
                 ("virtual_nccl_overlap", dict(vr=2, overlap=True)),
                 ("local_deep", dict(deep=True)), ("virtual_remote_deep", dict(vr=1, deep=True)),
                 ("virtual_nccl_deep", dict(vr=2, deep=True)),
                 ("virtual_lsa", dict(vr=3)), ("virtual_lsa_deep", dict(vr=3, deep=True))):
    ms, k = run(px, py, **kw)
    res[name] = {"ms": ms, "overhead": ms / one - 1.0, "kernels": k,
                 "over_serial_ideal": ms / (alone * px * py) - 1.0}
print(json.dumps(res), flush=True)
