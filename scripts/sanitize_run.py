"""Small workloads for compute-sanitizer (memcheck / racecheck / synccheck),
VERDICT r1 #8: bm 64^2 for 20 steps on one chunk, and a 2x2 local-chunk
fuzz deck for 2 steps (halo exchange + separate sweep kernels), both
checked against the oracle; 1x3 y strips with deep halos (deep), also
through the device-initiated store transport (lsa).
usage: sanitize_run.py [bm|chunks|deep|lsa]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from oracle import Oracle  # noqa: E402
from paper_conf_cluster_regulymg15_b200 import Clover  # noqa: E402
from workloads import bm_deck, fuzz_deck  # noqa: E402

case = sys.argv[1] if len(sys.argv) > 1 else "bm"
torch.cuda.set_device(0)
if case == "bm":
    deck, kw, steps = bm_deck(64), {}, 20
elif case in ("deep", "lsa"):
    # y strips with deep halos (row-shifted views), and the device-initiated
    # store transport (one-rank NCCL symmetric window)
    deck, kw, steps = fuzz_deck(9, nx=48, ny=64), dict(px=1, py=3), 3
else:
    deck, kw, steps = fuzz_deck(9, nx=48, ny=40), dict(px=2, py=2), 2
g = Clover(deck, **kw)
if case == "lsa":
    g.debug_set_virtual_remote(True, lsa=True)
if case in ("deep", "lsa"):
    assert g.deep_halo_active()
g.step(steps)
g.sync()
o = Oracle(deck)
o.step(steps)
for f in ("density0", "energy0", "xvel0", "yvel0"):
    assert np.array_equal(g.read(f), o.read(f)), f
g.field_summary()
g.close()
print("sanitize_run", case, "ok")
