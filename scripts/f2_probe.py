"""f2 probe A/B: per-kernel CUDA-event times at 3840^2 (bm)
with the production sweep-2 y kernel and with the probe kernel that also
evaluates the next step's viscosity + calc_dt terms.  Run twice, with
CLOVER_F2_PROBE=0 and =1 in the environment (read at clover_init)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_regulymg15_b200 import Clover  # noqa: E402
from workloads import bm_deck  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 3840
torch.cuda.set_device(0)
sim = Clover(bm_deck(n))
sim.step(20)
sim.sync()
prof = sim.profile_steps(40)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
e0.record(sim.stream)
sim.step(40)
e1.record(sim.stream)
torch.cuda.synchronize()
sim.sync()
print(json.dumps({"probe": os.environ.get("CLOVER_F2_PROBE", "0"), "mesh": n,
                  "ms_per_step_graphs": e0.elapsed_time(e1) / 40,
                  "kernels_ms": {k: v[0] / v[1] for k, v in prof.items()}}), flush=True)
