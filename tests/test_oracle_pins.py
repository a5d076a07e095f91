"""Pins of the CPU oracle against what the paper and the mathematics fix
(SURVEY.md 8(c) P1-P12).  CPU only (-m "not gpu").

The paper (sec. V) fixes the physics: the compressible Euler
equations as conservation laws of mass, momentum and energy on a structured
staggered grid.  The pins below check the oracle against consequences of that
which do NOT re-type the oracle's formulas: exact conservation, exact
symmetries, closed forms at t=0 and step 1, an exact Riemann solution, and
the reference code's recalled QA constant.
"""
from __future__ import annotations

import json
import math
import os

import numpy as np
import pytest

import riemann
from oracle import Oracle
from workloads import (bm_deck, colliding_slab_deck, contact_deck, doubled_deck, fuzz_deck, point_deck, quiescent_deck,
                       random_state_fields, sod_slab_deck, symmetric_deck, transpose_deck)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
GM1 = 0.4  # gamma - 1, mathematically (the oracle uses fp64 1.4-1.0)
STATE = ("density0", "energy0", "xvel0", "yvel0")


def _rel(a, b):
    return abs(a - b) / max(abs(a), abs(b))


# ---------------------------------------------------------------- P1
def test_p1_step0_summary_64():
    """Step-0 field_summary of bm64 (init painting + summary, c.1/c.12):
    32x13 state-2 cells (dyadic cell area, so vol/mass/ie are exact)."""
    o = Oracle(bm_deck(64))
    s = o.field_summary()
    area = (10.0 / 64) ** 2
    n2 = 32 * 13
    assert s["vol"] == 100.0
    assert s["mass"] == 0.2 * (4096 - n2) * area + 1.0 * n2 * area
    assert s["ie"] == 0.2 * 1.0 * (4096 - n2) * area + 1.0 * 2.5 * n2 * area
    assert s["ke"] == 0.0
    assert _rel(s["press"], GM1 * s["ie"]) < 1e-15


@pytest.mark.parametrize("n,block", [(960, (480, 192)), (200, (100, 40))])
def test_p1_step0_summary_large(n, block):
    o = Oracle(bm_deck(n))
    s = o.field_summary()
    area = (10.0 / n) ** 2
    n2 = block[0] * block[1]
    tol = n * n * 2.3e-16  # sequential-summation error bound n*eps
    assert _rel(s["vol"], 100.0) < tol
    assert _rel(s["mass"], 0.2 * 100 + 0.8 * n2 * area) < tol
    assert _rel(s["ie"], 0.2 * 100 + (2.5 - 0.2) * n2 * area) < tol
    assert s["ke"] == 0.0


# ---------------------------------------------------------------- P2
@pytest.mark.parametrize("n", [64, 240, 960])
def test_p2_first_dt_is_sound_speed_cfl(n):
    """First dt = min(0.7*dx/c2, 1.5*dtinit, dtmax) with the ideal-gas sound
    speed c = sqrt(gamma*(gamma-1)*e) of the hot state (fluid at rest, so the
    velocity and divergence limits are inactive)."""
    d = bm_deck(n)
    d["max_timestep"] = 1.0
    o = Oracle(d)
    dt = o.step(1)[0]
    dx = 10.0 / n
    expect = min(0.7 * dx / math.sqrt(1.4 * GM1 * 2.5), 1.5 * 0.04, 1.0)
    assert _rel(dt, expect) < 1e-14
    # capped deck
    o2 = Oracle(bm_deck(n))
    assert o2.step(1)[0] == min(dt, 0.04)


def test_p2_dt_rise_clamp():
    """dt may grow by at most dtrise per step (c.4 clamp)."""
    d = bm_deck(64)
    d["max_timestep"] = 10.0
    d["initial_timestep"] = 1e-3
    o = Oracle(d)
    dts = o.step(5)
    assert dts[0] == 1e-3 * 1.5
    for a, b in zip(dts[:-1], dts[1:]):
        assert b <= a * 1.5


# ---------------------------------------------------------------- P2c
@pytest.mark.parametrize("axis,factor", [("x", 0.35), ("y", 0.35), ("xy", 0.175)])
@pytest.mark.parametrize("n", [64, 72, 200])
def test_p2c_divergence_limit_binds_colliding_slabs(axis, factor, n):
    """c.4's divergence limit dtdivt = dtdiv_safe * (-1/div), div = net face
    volume flow / (2*volume), pinned in closed form.
    Colliding slabs at uniform pressure (q = 0 at step 1): the one column of
    cells whose left nodes move +U and right nodes -U has net outflow
    -4*U*dy per unit time, so div = -2U/dx and dtdivt = 0.7*dx/(2U) =
    0.35*dx/U; in the converging quadrants (xy) the centre cell adds the same
    from v: div = -4U/dx, dtdivt = 0.175*dx/U.  Every other limit is larger:
    the face-speed limit dtu = 0.5*dx/U, the sound-speed CFL 0.7*dx/c with
    c = sqrt(gamma*(gamma-1)*e) = sqrt(1.4) (U=1 > c/2), 1.5*dtinit = 0.06,
    dtmax = 1.  A dropped factor 2, a missing v (or u) term or a wrong sign
    of the divergence test changes the first dt by 2x or makes it negative."""
    U = 1.0
    o = Oracle(colliding_slab_deck(n, axis, U))
    dt = o.step(1)[0]
    dx = 10.0 / n
    c = math.sqrt(1.4 * GM1 * 2.5)
    expect = factor * dx / U
    others = (0.5 * dx / U, 0.7 * dx / c, 1.5 * 0.04, 1.0)
    assert expect < min(others) * 0.95  # the divergence term is the binding one
    assert _rel(dt, expect) < 1e-15


# ---------------------------------------------------------------- P3
@pytest.mark.parametrize("deck", [bm_deck(64, end_step=20), fuzz_deck(3), fuzz_deck(7),
                                  point_deck(64)])
def test_p3_conservation(deck):
    """Volume exact, mass conserved to round-off (flux form, reflective walls),
    press = (gamma-1)*ie to round-off (EOS identity)."""
    o = Oracle(deck)
    s0 = o.field_summary()
    ncell = deck["x_cells"] * deck["y_cells"]
    eps = 2.3e-16
    for _ in range(10):
        o.step(1)
        s = o.field_summary()
        assert s["vol"] == s0["vol"]
        assert _rel(s["mass"], s0["mass"]) < 1e-12
        # two sequential sums of ncell terms + 3 roundings per cell
        assert _rel(s["press"], GM1 * s["ie"]) < (ncell + 4) * eps


def test_p1_point_and_circle_painting():
    """generate_chunk's point and circle shapes: the point
    state covers exactly the one cell whose lower-left vertex is the point;
    a circle covers the cells whose centre lies within its radius (counted
    here from the cell-centre coordinates (j - 1/2) dx in closed form); a
    moving circle's velocity sits on exactly the corner nodes of its cells;
    the step-0 mass is the closed-form sum over the painted areas."""
    n = 64
    d = point_deck(n)
    o = Oracle(d)
    rho, e = o.read("density0"), o.read("energy0")
    u, v = o.read("xvel0"), o.read("yvel0")
    hot = np.argwhere(e == 20.0)
    assert hot.tolist() == [[n // 2, n // 2]]  # 0-based (k, j) of cell (33, 33)
    dx = 10.0 / n
    xc = (np.arange(1, n + 1) - 0.5) * dx  # exact on this dyadic mesh
    X, Y = np.meshgrid(xc, xc)
    dense = (X - 2.6) ** 2 + (Y - 7.3) ** 2 <= 1.1 ** 2
    light = (X - 7.2) ** 2 + (Y - 3.1) ** 2 <= 0.9 ** 2
    # no cell centre sits within rounding of either circle's edge
    for cx, cy, r in ((2.6, 7.3, 1.1), (7.2, 3.1, 0.9)):
        assert np.abs(np.hypot(X - cx, Y - cy) - r).min() > 1e-9
    assert np.array_equal(rho == 2.5, dense)
    assert np.array_equal(rho == 0.5, light)
    node = np.zeros((n + 1, n + 1), bool)
    for k, j in np.argwhere(light):
        node[k:k + 2, j:j + 2] = True
    assert np.array_equal(u == 0.3, node) and np.array_equal(v == -0.2, node)
    area = dx * dx
    n_dense, n_light = int(dense.sum()), int(light.sum())
    mass = (1.0 * (n * n - n_dense - n_light) + 2.5 * n_dense + 0.5 * n_light) * area
    assert _rel(o.field_summary()["mass"], mass) < 1e-14


def test_p3_total_energy_drift_small():
    o = Oracle(bm_deck(64))
    s0 = o.field_summary()
    o.step(20)
    s = o.field_summary()
    assert _rel(s["ie"] + s["ke"], s0["ie"]) < 5e-3


# ---------------------------------------------------------------- P4 / P4b
@pytest.mark.parametrize("rho,e", [(1.0, 2.5), (0.3, 1.7)])
def test_p4_quiescent_uniform_state_is_stationary(rho, e):
    o = Oracle(quiescent_deck(64, rho, e))
    before = {f: o.read(f) for f in STATE}
    dts = o.step(20)
    assert np.all(dts == dts[-1]) or np.all(np.diff(dts) >= 0)
    for f in STATE:
        a = o.read(f)
        if f in ("xvel0", "yvel0"):
            assert np.all(a == 0.0)
        else:
            assert np.all(a == a.flat[0])  # cell-to-cell uniform exactly
            if rho == 1.0:
                assert np.array_equal(a, before[f])


@pytest.mark.parametrize("centred", [False, True])
def test_p4b_contact_in_pressure_equilibrium_is_frozen(centred):
    """rho=1,e=1 | rho=0.5,e=2: p equal bitwise on both sides, so nothing
    moves; any spurious motion is a stencil/index bug."""
    o = Oracle(contact_deck(64, centred=centred))
    before = {f: o.read(f) for f in STATE}
    o.step(20)
    for f in STATE:
        assert np.array_equal(o.read(f), before[f]), f


# ---------------------------------------------------------------- P5
def test_p5_mirror_symmetry():
    """Centred square: x- and y-mirror symmetric to round-off."""
    o = Oracle(symmetric_deck(64))
    o.step(20)
    for f in STATE:
        a = o.read(f)
        sx = -1.0 if f == "xvel0" else 1.0
        sy = -1.0 if f == "yvel0" else 1.0
        scale = np.abs(a).max()
        assert np.abs(a - sx * a[:, ::-1]).max() <= 1e-13 * scale, f
        assert np.abs(a - sy * a[::-1, :]).max() <= 1e-13 * scale, f


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_p5_transpose_symmetry(seed):
    """Swapping x and y (and the first sweep direction) gives the transposed
    solution to round-off: pins every y-direction formula against its x twin."""
    d = fuzz_deck(seed)
    a, b = Oracle(d), Oracle(transpose_deck(d))
    da, db = a.step(10), b.step(10)
    assert np.abs(da - db).max() <= 1e-13 * da.max()
    pairs = (("density0", "density0"), ("energy0", "energy0"), ("xvel0", "yvel0"), ("yvel0", "xvel0"))
    for fa, fb in pairs:
        A, B = a.read(fa), b.read(fb).T
        assert np.abs(A - B).max() <= 1e-11 * np.abs(A).max(), fa


# ---------------------------------------------------------------- P6
def _slab_l1(nx):
    d = sod_slab_deck(nx, 4, max_timestep=0.04)
    o = Oracle(d)
    while o.clock()["time"] < 1.0:
        o.step(1)
    t = o.clock()["time"]
    rho = o.read("density0")
    v = o.read("yvel0")
    for r in range(1, rho.shape[0]):
        assert np.array_equal(rho[r], rho[0])  # every row identical
    assert np.all(v == 0.0)
    dx = 10.0 / nx
    xc = (np.arange(nx) + 0.5) * dx
    ex = riemann.sample(xc, t, 5.0, 1.0, 0.0, 1.0, 0.2, 0.0, 0.08)
    return np.abs(rho[0] - ex[0]).sum() * dx


@pytest.mark.slow
def test_p6_sod_slab_converges_to_exact_riemann_solution():
    errs = [_slab_l1(n) for n in (64, 128, 256)]
    assert errs[0] > errs[1] > errs[2]
    assert errs[2] < 0.06
    assert errs[0] / errs[2] > 2.0


def test_p6_star_state_textbook():
    p, u = riemann.star_state(1.0, 0.0, 1.0, 0.2, 0.0, 0.08)
    assert abs(p - 0.329011) < 2e-6 and abs(u - 0.868723) < 2e-6


# ---------------------------------------------------------------- P7
def test_p7_wall_normal_velocity_exactly_zero():
    o = Oracle(bm_deck(64))
    for _ in range(20):
        o.step(1)
        u = o.read("xvel0")
        v = o.read("yvel0")
        assert np.all(u[:, 0] == 0.0) and np.all(u[:, -1] == 0.0)
        assert np.all(v[0, :] == 0.0) and np.all(v[-1, :] == 0.0)


@pytest.mark.parametrize("seed", [0, 3, 6, 9])
def test_p7_wall_normal_velocity_zero_fuzz(seed):
    """Fuzz decks: zero to round-off (node-mass sums are accumulated in a
    fixed, not mirrored, order, so a wall can see ~1e-17)."""
    o = Oracle(fuzz_deck(seed))
    for _ in range(10):
        o.step(1)
        u, v = o.read("xvel0"), o.read("yvel0")
        tol = 1e-15 * max(np.abs(u).max(), np.abs(v).max())
        assert np.abs(u[:, 0]).max() <= tol and np.abs(u[:, -1]).max() <= tol
        assert np.abs(v[0, :]).max() <= tol and np.abs(v[-1, :]).max() <= tol


def test_a7_cellcentre_mirror_leaks_mass():
    """Reading A7 evidence: the cell-centre tangential face mirror lets mass
    through the walls on a deck with flow towards them, the geometric one
    conserves it (the equations are conservation laws)."""
    d = fuzz_deck(6)
    res = {}
    for fm in (0, 1):
        d["face_mirror"] = fm
        o = Oracle(d)
        m0 = o.field_summary()["mass"]
        o.step(10)
        res[fm] = _rel(o.field_summary()["mass"], m0)
    assert res[0] < 1e-13
    assert res[1] > 1e-9


# ---------------------------------------------------------------- P8
def test_p8_half_vs_doubled_domain():
    """bm on [0,10]^2 vs the mirrored problem on [-10,10]x[0,10]: the
    reflective wall at x=0 is an exact mirror, so the right half matches."""
    a = Oracle(bm_deck(64, face_mirror=0))
    b = Oracle(doubled_deck(64, 64, face_mirror=0))
    a.step(20)
    b.step(20)
    for f in STATE:
        A, B = a.read(f), b.read(f)
        half = B[:, B.shape[1] - A.shape[1]:]
        assert np.abs(A - half).max() <= 1e-13 * np.abs(A).max(), f


# ---------------------------------------------------------------- P10
@pytest.mark.slow
def test_p10_qa_constant_clover_bm_short():
    with open(os.path.join(GOLDEN, "qa_bm_short.json")) as fh:
        g = json.load(fh)
    o = Oracle(bm_deck(g["x_cells"]))
    o.step(g["steps"])
    ke = o.field_summary()["ke"]
    qa_diff = abs(100.0 * (ke / g["ke"]) - 100.0)
    assert qa_diff < g["rel_tol_percent"]
    assert qa_diff < 1e-9  # observed: ~1e-13 %


# ---------------------------------------------------------------- P11
def test_p11_trend():
    o = Oracle(bm_deck(64))
    ke, ie = [], []
    for _ in range(20):
        o.step(1)
        s = o.field_summary()
        ke.append(s["ke"])
        ie.append(s["ie"])
    assert all(b > a for a, b in zip(ke, ke[1:]))
    assert all(b < a for a, b in zip(ie, ie[1:]))


# ---------------------------------------------------------------- P12
def test_p12_step1_lagrangian_closed_forms():
    """Step 1 from rest: PdV predictor leaves rho, e unchanged; accelerate
    gives u1 = dt*(p2-p1)/(m_node/...) on the state-2 edge nodes."""
    n = 64
    o = Oracle(bm_deck(n))
    rho0, e0 = o.read("density0"), o.read("energy0")
    assert o.run_stage("timestep") == 0
    dt = o.clock()["dt"]
    assert dt == 0.04
    assert np.all(o.read("viscosity") == 0.0)
    o.run_stage("pdv_predict")
    assert np.array_equal(o.read("density1"), rho0)
    assert np.array_equal(o.read("energy1"), e0)
    o.run_stage("accelerate")
    u1, v1 = o.read("xvel1"), o.read("yvel1")
    dx = 10.0 / n
    dp = GM1 * 1.0 * 2.5 - GM1 * 0.2 * 1.0
    edge = dt * dp / (0.6 * dx)
    corner = dt * dp / (0.8 * dx)
    # vertical edge x=5 is node column j=33 (index 32), rows k=2..13 interior of the edge
    for k in range(2, 14):
        assert _rel(u1[k - 1, 32], edge) < 1e-14
        assert v1[k - 1, 32] == 0.0
    # horizontal edge y=2.03 is node row k=14 (index 13)
    for j in range(2, 33):
        assert _rel(v1[13, j - 1], edge) < 1e-14
    assert _rel(u1[13, 32], corner) < 1e-14 and _rel(v1[13, 32], corner) < 1e-14
    # left wall: u = 0, v tangential carries the edge value
    assert u1[13, 0] == 0.0 and _rel(v1[13, 0], edge) < 1e-14
    # nodes away from the state-2 boundary do not move
    mask = np.ones_like(u1, bool)
    mask[:15, :34] = False
    assert np.all(u1[mask] == 0.0) and np.all(v1[mask] == 0.0)


def test_fuzz_decks_run_and_conserve():
    for seed in range(4):
        d = fuzz_deck(seed)
        o = Oracle(d)
        m0 = o.field_summary()["mass"]
        o.step(5)
        assert _rel(o.field_summary()["mass"], m0) < 1e-12


def test_random_state_roundtrip():
    o = Oracle(bm_deck(16))
    f = random_state_fields(1, 16, 16)
    o.load_state(f)
    for k, v in f.items():
        assert np.array_equal(o.read(k), v)


def test_compensated_summary_is_exact_on_dyadic_mesh_and_close_elsewhere():
    """Both summations of c.12: bitwise equal where every term and partial
    sum is exact (64^2 bm, dyadic); within the sequential bound n*eps on
    960^2, where the compensated sum also matches the closed form closer."""
    o = Oracle(bm_deck(64))
    assert o.field_summary() == o.field_summary(compensated=True)
    o = Oracle(bm_deck(960))
    a, b = o.field_summary(), o.field_summary(compensated=True)
    for k in a:
        if b[k]:
            assert _rel(a[k], b[k]) < 960 * 960 * 2.3e-16
    assert _rel(b["vol"], 100.0) < 1e-14 < _rel(a["vol"], 100.0)
