"""Per-kernel CUDA-event times (clover_profile_steps) and the graph step time
of one chunk of NX x NY (bm deck, square cells), after 20 warm-up steps.
usage: kernel_times.py NX NY [STEPS] [active]  -> one JSON line
active: a seeded smooth random state on every cell (workloads.random_state_fields),
so the per-cell work does not depend on how far the bm shock has travelled."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_regulymg15_b200 import Clover  # noqa: E402
from workloads import bm_deck  # noqa: E402

nx, ny = int(sys.argv[1]), int(sys.argv[2])
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 40
active = len(sys.argv) > 4 and sys.argv[4] == "active"
torch.cuda.set_device(0)
deck = bm_deck(nx, ny, xmax=10.0, ymax=10.0 * ny / nx)
if active:
    from workloads import random_state_fields
    deck["max_timestep"] = 1.0
sim = Clover(deck)
if active:
    sim.load_state(random_state_fields(7, nx, ny, smooth=True))
sim.step(20)
sim.sync()
prof = sim.profile_steps(steps)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
e0.record(sim.stream)
sim.step(steps)
e1.record(sim.stream)
torch.cuda.synchronize()
sim.sync()
ms = e0.elapsed_time(e1) / steps
print(json.dumps({"mesh": [nx, ny], "active": active, "ms_per_step_graphs": ms, "ns_per_cell": ms * 1e6 / (nx * ny),
                  "kernels_ms": {k: v[0] / v[1] for k, v in prof.items()},
                  "profiled_ms_per_step": sum(v[0] for v in prof.values()) / steps}), flush=True)
