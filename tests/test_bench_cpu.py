"""CPU checks of bench.py's workload selection (no GPU): the arm's mesh for
each N (configs[2], the A4 weak series, --strong, --mesh) and the reference
arm's bounded sample of that same workload (same width and cell size)."""
from __future__ import annotations

import argparse
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def _args(strong=False, mesh=None):
    return argparse.Namespace(strong=strong, mesh=mesh)


@pytest.mark.parametrize("world,expect", [(1, (3840, 3840, 1, 1)), (2, (7680, 3840, 1, 2)),
                                          (4, (7680, 7680, 1, 4)), (8, (15360, 7680, 1, 8))])
def test_arm_mesh_weak_series(world, expect):
    assert bench.arm_mesh(_args(), world) == expect


def test_arm_mesh_strong_and_override():
    assert bench.arm_mesh(_args(strong=True), 8)[:2] == (7680, 7680)
    assert bench.arm_mesh(_args(mesh=[960, 480]), 1)[:2] == (960, 480)


@pytest.mark.parametrize("nx,ny,rows", [(3840, 3840, 240), (15360, 7680, 60), (7680, 7680, 120)])
def test_reference_band_has_the_arm_cell_size(nx, ny, rows):
    d = bench.band_deck(nx, ny, rows)
    assert (d["x_cells"], d["y_cells"]) == (nx, rows)
    dx = (d["xmax"] - d["xmin"]) / d["x_cells"]
    dy = (d["ymax"] - d["ymin"]) / d["y_cells"]
    assert dx == pytest.approx(10.0 / nx, rel=1e-15)
    assert dy == pytest.approx(10.0 / ny, rel=1e-15)
