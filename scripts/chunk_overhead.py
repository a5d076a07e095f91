"""Cost of the halo-exchange machinery on one GPU: the same bm mesh as one
chunk and as px x py local chunks (device-to-device exchange phases), and
through the virtual-remote packing path (pack -> staging -> unpack, the
multi-GPU message layout).  usage: chunk_overhead.py NX NY PX PY [STEPS]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_regulymg15_b200 import Clover  # noqa: E402
from paper_conf_cluster_regulymg15_b200.clover import load  # noqa: E402
from workloads import bm_deck  # noqa: E402

nx, ny, px, py = (int(a) for a in sys.argv[1:5])
steps = int(sys.argv[5]) if len(sys.argv) > 5 else 20
torch.cuda.set_device(0)
deck = bm_deck(nx, ny, end_step=steps, ymax=10.0 * ny / nx)


def run(p, q, vr=False):
    sim = Clover(deck, px=p, py=q)
    if vr:
        load().clover_debug_set_virtual_remote(sim._ctx, 1)
    sim.step(3)
    sim.sync()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(sim.stream)
    sim.step(steps)
    e1.record(sim.stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    sim.close()
    return ms


one = run(1, 1)
many = run(px, py)
vr = run(px, py, True)
print(f"{nx}x{ny}: 1 chunk {one:.4f} ms/step; {px}x{py} local chunks {many:.4f} ms/step "
      f"(+{many - one:.4f}); virtual remote {vr:.4f} (+{vr - one:.4f})")
