"""Fixed workload for ncu captures: bm deck, direct launches (no graphs) so
every kernel is a separate named launch.  usage: prof_run.py NX NY STEPS"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cluster_regulymg15_b200 import Clover  # noqa: E402
from workloads import bm_deck  # noqa: E402

nx, ny, steps = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
torch.cuda.set_device(0)
sim = Clover(bm_deck(nx, ny))
sim.set_graphs(False)
sim.step(steps)
sim.sync()
print("done", sim.clock())
