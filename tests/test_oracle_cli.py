"""The oracle's I/O contract: the command-line driver
reads the reference's text deck, prints the step log and summaries as JSON
lines with round-trip exact doubles, and dumps every field's global interior
as raw fp64 in the clover_read_field layout.  CPU only; the GPU byte
compare against these dumps is in test_gpu_parity.py."""
from __future__ import annotations

import json
import os
import subprocess

import numpy as np
import pytest

import oracle
from oracle import Oracle, field_shape
from oracle.deck import deck_to_text, parse_text_deck
from workloads import bm_deck, fuzz_deck, point_deck

# SURVEY 8(c) c.15's deck, verbatim (the bm problem on 64^2, 20 steps)
SURVEY_DECK = """*clover
 state 1 density=0.2 energy=1.0
 state 2 density=1.0 energy=2.5 geometry=rectangle xmin=0.0 xmax=5.0 ymin=0.0 ymax=2.0
 x_cells=64  y_cells=64  xmin=0.0 ymin=0.0 xmax=10.0 ymax=10.0
 initial_timestep=0.04  max_timestep=0.04  timestep_rise=1.5  end_step=20
*endclover
"""
FIELDS = ("density0", "energy0", "pressure", "viscosity", "soundspeed", "xvel0", "yvel0",
          "vol_flux_x", "vol_flux_y", "mass_flux_x", "mass_flux_y")


def run_cli(tmp_path, text, *args):
    oracle.build()
    p = tmp_path / "clover.in"
    p.write_text(text)
    r = subprocess.run([oracle.CLI_PATH, *args, str(p)], capture_output=True, text=True, timeout=300)
    lines = [json.loads(x) for x in r.stdout.splitlines() if x.strip()]
    return r.returncode, lines, r.stderr


def test_survey_deck_step_log_and_closed_form_summary(tmp_path):
    rc, lines, err = run_cli(tmp_path, SURVEY_DECK, "--summary-every", "10")
    assert rc == 0, err
    steps = [x for x in lines if "step" in x]
    sums = [x for x in lines if "summary" in x]
    assert [x["step"] for x in steps] == list(range(1, 21))
    assert [x["summary"] for x in sums] == [0, 10, 20]
    # P1 closed form at step 0 (32x13 state-2 cells on the dyadic 64^2 mesh)
    area = (10.0 / 64) ** 2
    s0 = sums[0]
    assert s0["vol"] == 100.0 and s0["ke"] == 0.0
    assert s0["mass"] == 0.2 * (4096 - 416) * area + 1.0 * 416 * area
    assert s0["density"] == s0["mass"] / s0["vol"] and s0["total"] == s0["ie"] + s0["ke"]
    # the dt history is exactly the library's (%.17g round-trips), and the
    # capped bm deck keeps dt = 0.04
    dts = Oracle(bm_deck(64)).step(20)
    assert np.array_equal(np.array([x["dt"] for x in steps]), dts)
    assert all(x["dt"] == 0.04 for x in steps)


def test_dump_matches_read_field_layout(tmp_path):
    deck = fuzz_deck(4, nx=37, ny=29)
    rc, lines, err = run_cli(tmp_path, deck_to_text(deck), "--steps", "5", "--dump", str(tmp_path))
    assert rc == 0, err
    o = Oracle(deck)
    o.step(5)
    o.field_summary()  # the driver's last summary refreshes p and cs from the state (c.12)
    for f in FIELDS:
        a = np.fromfile(tmp_path / f"{f}.f64", dtype="<f8").reshape(field_shape(f, 37, 29))
        assert np.array_equal(a, o.read(f)), f


@pytest.mark.parametrize("deck", [bm_deck(64), fuzz_deck(3), point_deck(48, 40),
                                  dict(fuzz_deck(5), face_mirror=1, advect_x_first=0)])
def test_text_deck_round_trip_and_same_run(tmp_path, deck):
    back = parse_text_deck(deck_to_text(deck))
    for k in ("x_cells", "y_cells", "xmin", "ymin", "xmax", "ymax", "initial_timestep",
              "max_timestep", "face_mirror", "advect_x_first"):
        assert back.get(k, {"face_mirror": 0}.get(k)) == deck.get(k, {"face_mirror": 0}.get(k)), k
    assert len(back["states"]) == len(deck["states"])
    for a, b in zip(back["states"], deck["states"]):
        for k in ("density", "energy", "xvel", "yvel", "xmin", "xmax", "ymin", "ymax", "radius"):
            assert a.get(k, 0.0) == b.get(k, 0.0), k
    rc, lines, err = run_cli(tmp_path, deck_to_text(deck), "--steps", "6")
    assert rc == 0, err
    dts = np.array([x["dt"] for x in lines if "step" in x])
    assert np.array_equal(dts, Oracle(deck).step(6))


def test_bad_decks_are_rejected(tmp_path):
    assert run_cli(tmp_path, "x_cells=4\n")[0] == 2                       # no *clover block
    assert run_cli(tmp_path, "*clover\n x_cells=8\n*endclover\n")[0] == 2  # no states
    bad = SURVEY_DECK.replace("geometry=rectangle", "geometry=hexagon")
    assert run_cli(tmp_path, bad)[0] == 2
    assert run_cli(tmp_path, SURVEY_DECK.replace("x_cells=64", "x_cells=six"))[0] == 2


def test_small_dt_exit_status(tmp_path):
    rc, lines, _ = run_cli(tmp_path, SURVEY_DECK.replace("end_step=20", "end_step=3 dtmin=0.5"))
    assert rc == 5
    assert not [x for x in lines if "step" in x]
