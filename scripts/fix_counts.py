"""Flagged warp segments (IEEE fixup redos) per step on bm 3840^2 over the
300-step run: cumulative count from clover_debug_fix_count at checkpoints."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_regulymg15_b200 import Clover  # noqa: E402
from workloads import bm_deck  # noqa: E402

torch.cuda.set_device(0)
sim = Clover(bm_deck(3840))
done, prev, out = 0, 0, []
for s in (5, 55, 100, 200, 300):
    sim.step(s - done)
    sim.sync()
    n = sim.debug_fix_count()
    out.append({"steps": [done + 1, s], "flagged_segments": n - prev, "per_step": (n - prev) / (s - done)})
    done, prev = s, n
print(json.dumps(out))
