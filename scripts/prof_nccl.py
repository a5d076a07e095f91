"""Workload for the ncu launch list of the NCCL virtual-remote mode (VERDICT
r1 #4): fuzz deck 96x80 on 2x2 chunks, every chunk boundary through a
one-rank NCCL communicator (ncclSend/ncclRecv to self + ncclAllReduce MIN),
direct launches; checked bitwise against one chunk."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_regulymg15_b200 import Clover  # noqa: E402
from workloads import fuzz_deck  # noqa: E402

torch.cuda.set_device(0)
deck = fuzz_deck(9, nx=96, ny=80)
one = Clover(deck)
many = Clover(deck, px=2, py=2)
many.debug_set_virtual_remote(True, nccl=True)
many.set_graphs(False)
one.step(2)
many.step(2)
for f in ("density0", "energy0", "xvel0", "yvel0"):
    assert np.array_equal(one.read(f), many.read(f)), f
print("nccl virtual 2x2 ok")
