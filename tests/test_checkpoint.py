"""Checkpoint/restart (sec. VI / Fig. 8; SURVEY 8(f)
f3).  CPU: the library's access-execute checkpoint plan is validated
against the oracle's actual data flow -- zeroing every dataset the plan drops
at a loop boundary must leave the run bit-identical.  GPU: checkpoint at a
step boundary and restart continue bit for bit."""
from __future__ import annotations

import numpy as np
import pytest

from oracle import Oracle, field_shape
from paper_conf_cluster_regulymg15_b200.clover import CKPT_DATASETS, checkpoint_plan
from workloads import bm_deck, fuzz_deck

STATE = ("density0", "energy0", "xvel0", "yvel0")
# oracle stage boundaries -> index of the loop that follows (clover_checkpoint_plan numbering)
BOUNDARIES = [("timestep", 3), ("pdv_predict", 5), ("accelerate", 6), ("pdv_correct", 7),
              ("flux_calc", 8), ("adv_cell1", 9), ("adv_mom1", 10), ("adv_cell2", 11),
              ("adv_mom2", 12)]
STAGES = ["timestep", "pdv_predict", "accelerate", "pdv_correct", "flux_calc", "adv_cell1",
          "adv_mom1", "adv_cell2", "adv_mom2", "reset"]


def test_plan_minimum_is_the_step_boundary():
    counts = {}
    for loop in range(13):
        name, save = checkpoint_plan(loop)
        counts[loop] = len(save)
    assert checkpoint_plan(0) == ("ideal_gas", list(STATE))
    assert min(counts.values()) == 4
    assert [l for l, n in counts.items() if n == 4] == [0, 12]
    assert checkpoint_plan(12)[1] == ["density1", "energy1", "xvel1", "yvel1"]


def _run_with_dropped(deck, steps_before, boundary, drop):
    o = Oracle(deck)
    o.step(steps_before)
    for st in STAGES:
        o.run_stage(st)
        if st == boundary:
            for name in drop:
                o.write(name, np.zeros(field_shape(name, o.nx, o.ny)))
    o.step(2)
    return o


@pytest.mark.parametrize("boundary,loop", BOUNDARIES)
def test_plan_is_sufficient_against_the_oracle(boundary, loop):
    deck = fuzz_deck(4)
    _, save = checkpoint_plan(loop)
    drop = [d for d in CKPT_DATASETS if d not in save]
    ref = _run_with_dropped(deck, 3, boundary, [])
    got = _run_with_dropped(deck, 3, boundary, drop)
    for f in STATE:
        assert np.array_equal(ref.read(f), got.read(f)), (boundary, f)


def test_dropping_a_saved_dataset_changes_the_result():
    """the plan is not vacuous: zeroing a dataset it keeps does matter."""
    deck = fuzz_deck(4)
    ref = _run_with_dropped(deck, 3, "flux_calc", [])
    got = _run_with_dropped(deck, 3, "flux_calc", ["vol_flux_x"])
    assert not np.array_equal(ref.read("density0"), got.read("density0"))


@pytest.mark.gpu
def test_gpu_checkpoint_restart_bitwise():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_cluster_regulymg15_b200 import Clover
    deck = bm_deck(96, 64)
    a = Clover(deck)
    a.step(7)
    blob = a.checkpoint()
    a.step(9)
    b = Clover(deck)
    b.restart(blob)
    assert b.clock()["step"] == 7
    b.step(9)
    for f in STATE:
        assert np.array_equal(a.read(f), b.read(f)), f
    assert a.clock() == b.clock()
    assert np.array_equal(a.dt_history(8, 9), b.dt_history(8, 9))
    # steps before the restart point are not in b's history
    from paper_conf_cluster_regulymg15_b200 import CloverError
    with pytest.raises(CloverError):
        b.dt_history(7, 2)
    # restart into a context that has already run a different history
    c = Clover(deck)
    c.step(3)
    c.restart(blob)
    c.step(9)
    for f in STATE:
        assert np.array_equal(a.read(f), c.read(f)), f
    # and the oracle agrees with the continued run
    o = Oracle(deck)
    o.step(16)
    for f in STATE:
        assert np.array_equal(a.read(f), o.read(f)), f


@pytest.mark.gpu
def test_gpu_checkpoint_across_decompositions_with_deep_halos():
    """A checkpoint is the global state: taken on one chunk, restarted on 1x4
    y strips with deep halos (the restart refreshes the state halo 7 rows
    deep), and back; the continued runs stay bitwise equal to one chunk."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_cluster_regulymg15_b200 import Clover
    deck = bm_deck(96, 128)
    one = Clover(deck)
    one.step(6)
    blob = one.checkpoint()
    one.step(8)
    strips = Clover(deck, px=1, py=4)
    assert strips.deep_halo_active()
    strips.restart(blob)
    strips.step(5)
    blob2 = strips.checkpoint()
    strips.step(3)
    back = Clover(deck)
    back.restart(blob2)
    back.step(3)
    for f in STATE:
        assert np.array_equal(strips.read(f), one.read(f)), f
        assert np.array_equal(back.read(f), one.read(f)), f
    assert np.array_equal(strips.dt_history(7, 8), one.dt_history(7, 8))


@pytest.mark.gpu
def test_gpu_restart_rejects_other_mesh():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_cluster_regulymg15_b200 import Clover, CloverError
    a = Clover(bm_deck(64))
    blob = a.checkpoint()
    b = Clover(bm_deck(48))
    with pytest.raises(CloverError):
        b.restart(blob)
    with pytest.raises(CloverError):
        a.restart(b"\0" * len(blob))
