"""Full-size parity run (test infrastructure, not the product path): the bm
deck at a BASELINE config size through the production launch configuration
(graphs, one chunk), against the CPU oracle on the same deck for the same
number of steps.  Compares every state field bit for bit, the dt history bit
for bit and the field summary (1e-10 relative against the oracle's
compensated sum, A15/A17).

usage: python scripts/validate_full.py NX NY STEPS [OUT.json]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from oracle import Oracle  # noqa: E402
from paper_conf_cluster_regulymg15_b200 import Clover  # noqa: E402
from workloads import bm_deck  # noqa: E402

nx, ny, steps = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
out = sys.argv[4] if len(sys.argv) > 4 else None
deck = bm_deck(nx, ny, end_step=steps, ymax=10.0 * ny / nx)
torch.cuda.set_device(0)
t0 = time.perf_counter()
g = Clover(deck)
g.step(steps)
g.sync()
tg = time.perf_counter() - t0
t0 = time.perf_counter()
o = Oracle(deck)
dts = o.step(steps)
to = time.perf_counter() - t0
res = {"mesh": [nx, ny], "steps": steps, "gpu_s": tg, "oracle_s": to,
       "dt_history_bitwise": bool(np.array_equal(g.dt_history(1, steps), dts)), "fields": {}}
ok = res["dt_history_bitwise"]
for f in ("density0", "energy0", "xvel0", "yvel0"):
    a, b = g.read(f), o.read(f)
    nd = int((a != b).sum())
    res["fields"][f] = {"elements": int(a.size), "differ": nd,
                        "max_abs_diff": float(np.abs(a - b).max())}
    ok &= nd == 0
gs = g.field_summary()
osm = o.field_summary(compensated=True)
res["summary_rel"] = {k: (abs(gs[k] - osm[k]) / abs(osm[k]) if osm[k] else abs(gs[k]))
                      for k in ("vol", "mass", "ie", "ke", "press")}
ok &= all(v <= 1e-10 for v in res["summary_rel"].values())
res["clock"] = g.clock()
res["pass"] = bool(ok)
print(json.dumps(res))
if out:
    with open(out, "w") as fh:
        json.dump(res, fh, indent=1)
sys.exit(0 if ok else 1)
