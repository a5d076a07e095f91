"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests,
bench.py and smoke().

This module holds NO arithmetic of the method: it only builds input decks
(mesh + state list) and seeded random field arrays.  Both
the oracle (oracle/) and the CUDA path (paper_conf_cluster_regulymg15_b200/)
consume its output; neither is imported here.

Decks are plain dicts:
  {"x_cells", "y_cells", "xmin", "ymin", "xmax", "ymax",
   "initial_timestep", "max_timestep", "timestep_rise", "end_step",
   "advect_x_first", "face_mirror", "states": [ {density, energy, xvel, yvel,
   geometry, xmin, xmax, ymin, ymax, radius}, ... ]}
states[0] is the background state (fills every cell).
"""
from __future__ import annotations

import copy

import numpy as np

GEOM = {"rectangle": 1, "circle": 2, "point": 3}

# Reading A7: tangential mirror of face fields at walls.
FACE_MIRROR_GEOMETRIC = 0
FACE_MIRROR_CELLCENTRE = 1
DEFAULT_FACE_MIRROR = FACE_MIRROR_GEOMETRIC  # DESIGN.md reading A7


def _state(density, energy, xvel=0.0, yvel=0.0, geometry="rectangle",
           xmin=0.0, xmax=0.0, ymin=0.0, ymax=0.0, radius=0.0):
    return dict(density=float(density), energy=float(energy), xvel=float(xvel),
                yvel=float(yvel), geometry=geometry, xmin=float(xmin),
                xmax=float(xmax), ymin=float(ymin), ymax=float(ymax),
                radius=float(radius))


def bm_deck(nx: int = 960, ny: int | None = None, end_step: int = 87, **kw):
    """The two-state benchmark deck (clover_bm shape; SURVEY 8(c) A3, 8(d)
    C1-C5): state 1 rho=0.2 e=1.0 background, state 2 rho=1.0 e=2.5 on the
    rectangle [0,5]x[0,2], domain [0,10]^2, dtinit=dtmax=0.04, rise 1.5."""
    ny = nx if ny is None else ny
    d = dict(x_cells=int(nx), y_cells=int(ny), xmin=0.0, ymin=0.0, xmax=10.0,
             ymax=10.0, initial_timestep=0.04, max_timestep=0.04,
             timestep_rise=1.5, end_step=int(end_step), advect_x_first=1,
             face_mirror=DEFAULT_FACE_MIRROR,
             states=[_state(0.2, 1.0),
                     _state(1.0, 2.5, geometry="rectangle", xmin=0.0, xmax=5.0,
                            ymin=0.0, ymax=2.0)])
    d.update(kw)
    return d


def symmetric_deck(n: int = 64, end_step: int = 20, **kw):
    """Centred-square variant of bm: state 2 on [3.75,6.25]^2,
    mirror-symmetric about x=5 and y=5."""
    d = bm_deck(n, n, end_step, **kw)
    d["states"][1].update(xmin=3.75, xmax=6.25, ymin=3.75, ymax=6.25)
    return d


def point_deck(nx: int = 64, ny: int | None = None, end_step: int = 20, jp: int | None = None,
               kp: int | None = None):
    """Geometry deck (the reference's circle and point state
    shapes): background rho=1 e=1; a point state (rho=1, e=20) painted on the
    one cell whose lower-left vertex is the point, placed on vertex (jp, kp)
    (1-based; default the domain centre) with the vertex coordinate computed
    as generate_chunk does, xmin + dx*(jp-1); a resting dense circle
    (rho=2.5, e=0.5, r=1.1 about (2.6, 7.3)) and a moving light circle
    (rho=0.5, e=1.5, u=0.3, v=-0.2, r=0.9 about (7.2, 3.1)), both clear of the
    walls (reading A16)."""
    ny = nx if ny is None else ny
    d = bm_deck(nx, ny, end_step)
    d["max_timestep"] = 0.04
    jp = nx // 2 + 1 if jp is None else jp
    kp = ny // 2 + 1 if kp is None else kp
    dx, dy = (10.0 - 0.0) / float(nx), (10.0 - 0.0) / float(ny)
    px, py = 0.0 + dx * float(jp - 1), 0.0 + dy * float(kp - 1)
    d["states"] = [_state(1.0, 1.0),
                   _state(2.5, 0.5, geometry="circle", xmin=2.6, ymin=7.3, radius=1.1),
                   _state(0.5, 1.5, 0.3, -0.2, geometry="circle", xmin=7.2, ymin=3.1, radius=0.9),
                   _state(1.0, 20.0, geometry="point", xmin=px, ymin=py)]
    return d


def quiescent_deck(n: int = 64, density=1.0, energy=2.5, end_step: int = 20):
    """One uniform state at rest."""
    d = bm_deck(n, n, end_step)
    d["states"] = [_state(density, energy)]
    return d


def contact_deck(n: int = 64, end_step: int = 20, centred: bool = False):
    """Stationary contact in exact pressure equilibrium:
    rho=1 e=1 | rho=0.5 e=2, so p=(GM1*rho)*e is bitwise equal on both sides."""
    d = bm_deck(n, n, end_step)
    box = dict(xmin=3.75, xmax=6.25, ymin=3.75, ymax=6.25) if centred else \
        dict(xmin=0.0, xmax=5.0, ymin=0.0, ymax=10.0)
    d["states"] = [_state(1.0, 1.0), _state(0.5, 2.0, geometry="rectangle", **box)]
    return d


def sod_slab_deck(nx: int = 256, ny: int = 4, end_step: int = 100, max_timestep=0.04):
    """1D Sod-type slab along x: left rho=1 p=1, right rho=0.2
    p=0.08 (gamma=1.4 -> e = p/((gamma-1) rho)): e_L=2.5, e_R=1.0."""
    d = bm_deck(nx, ny, end_step)
    d["ymax"] = 10.0 * ny / nx  # square cells
    d["max_timestep"] = max_timestep
    d["states"] = [_state(0.2, 1.0),
                   _state(1.0, 2.5, geometry="rectangle", xmin=0.0, xmax=5.0,
                          ymin=0.0, ymax=d["ymax"])]
    return d


def colliding_slab_deck(n: int = 64, axis: str = "x", U: float = 1.0, end_step: int = 10):
    """Colliding slabs (pins calc_dt's divergence term,
    SURVEY 8(c) c.4): uniform rho=1, e=2.5 (so p is uniform and q = 0 at
    step 1); along `axis`, a slab on [3,5] moves with +U and a slab on [5,7]
    with -U across the whole other axis.  axis="xy": four quadrants of
    [3,7]^2 converge on (5,5) (u = +-U and v = +-U).  dtinit 0.04 (x1.5 =
    0.06), dtmax 1.0, so the first dt is min(dtdiv, dtu, dtc), with U > c/2
    making the divergence limit the binding one."""
    d = bm_deck(n, n, end_step)
    d["max_timestep"] = 1.0
    bg = _state(1.0, 2.5)
    if axis == "x":
        d["states"] = [bg, _state(1.0, 2.5, U, 0.0, xmin=3.0, xmax=5.0, ymin=0.0, ymax=10.0),
                       _state(1.0, 2.5, -U, 0.0, xmin=5.0, xmax=7.0, ymin=0.0, ymax=10.0)]
    elif axis == "y":
        d["states"] = [bg, _state(1.0, 2.5, 0.0, U, xmin=0.0, xmax=10.0, ymin=3.0, ymax=5.0),
                       _state(1.0, 2.5, 0.0, -U, xmin=0.0, xmax=10.0, ymin=5.0, ymax=7.0)]
    elif axis == "xy":
        d["states"] = [bg,
                       _state(1.0, 2.5, U, U, xmin=3.0, xmax=5.0, ymin=3.0, ymax=5.0),
                       _state(1.0, 2.5, -U, U, xmin=5.0, xmax=7.0, ymin=3.0, ymax=5.0),
                       _state(1.0, 2.5, U, -U, xmin=3.0, xmax=5.0, ymin=5.0, ymax=7.0),
                       _state(1.0, 2.5, -U, -U, xmin=5.0, xmax=7.0, ymin=5.0, ymax=7.0)]
    else:
        raise ValueError(axis)
    return d


def doubled_deck(nx_half: int = 64, ny: int = 64, end_step: int = 20, **kw):
    """bm mirrored about x=0: domain [-10,10]x[0,10] on
    (2*nx_half) x ny, state 2 on [-5,5]x[0,2]."""
    d = bm_deck(2 * nx_half, ny, end_step, **kw)
    d["xmin"] = -10.0
    d["states"][1].update(xmin=-5.0, xmax=5.0)
    return d


def transpose_deck(deck):
    """Swap the roles of x and y (mesh, domain, states, velocities)."""
    d = copy.deepcopy(deck)
    d["x_cells"], d["y_cells"] = deck["y_cells"], deck["x_cells"]
    d["xmin"], d["ymin"] = deck["ymin"], deck["xmin"]
    d["xmax"], d["ymax"] = deck["ymax"], deck["xmax"]
    d["advect_x_first"] = 0 if deck.get("advect_x_first", 1) else 1
    for s, s0 in zip(d["states"], deck["states"]):
        s["xmin"], s["ymin"] = s0["ymin"], s0["xmin"]
        s["xmax"], s["ymax"] = s0["ymax"], s0["xmax"]
        s["xvel"], s["yvel"] = s0["yvel"], s0["xvel"]
    return d


def fuzz_deck(seed: int, nx: int | None = None, ny: int | None = None,
              nstates: int = 4, end_step: int = 10):
    """Seeded random multi-state deck: random mesh (unless given),
    random rectangle/circle states with random density/energy/velocity.
    numpy PCG64 seeded generator.  State geometry stays inside [2,8]^2 so no
    moving state touches a wall node (reading A16: wall-normal velocity must
    start at zero for the reflective walls to conserve mass)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    nx = int(rng.integers(8, 48)) if nx is None else nx
    ny = int(rng.integers(8, 48)) if ny is None else ny
    d = bm_deck(nx, ny, end_step)
    d["max_timestep"] = 1.0
    states = [_state(rng.uniform(0.2, 1.0), rng.uniform(0.5, 2.5))]
    for _ in range(nstates - 1):
        x0, x1 = np.sort(rng.uniform(2.0, 8.0, 2))
        y0, y1 = np.sort(rng.uniform(2.0, 8.0, 2))
        geom = "rectangle" if rng.uniform() < 0.7 else "circle"
        if geom == "circle":  # centre (xmin, ymin) in [3,7]^2, radius <= 1.5
            x0, y0 = rng.uniform(3.0, 7.0, 2)
        states.append(_state(rng.uniform(0.1, 2.0), rng.uniform(0.3, 3.0),
                             rng.uniform(-0.5, 0.5), rng.uniform(-0.5, 0.5),
                             geometry=geom, xmin=x0, xmax=x1, ymin=y0, ymax=y1,
                             radius=rng.uniform(0.5, 1.5)))
    d["states"] = states
    return d


def random_state_fields(seed: int, nx: int, ny: int, smooth: bool = False,
                        wall_velocity: bool = False):
    """Seeded random-but-physical state (density0, energy0 on cells;
    xvel0, yvel0 on nodes), global interior layout, row-major j fastest.
    White noise by default so every limiter branch fires."""
    rng = np.random.Generator(np.random.PCG64(seed))
    shape_c = (ny, nx)
    shape_n = (ny + 1, nx + 1)
    rho = rng.uniform(0.2, 2.0, shape_c)
    e = rng.uniform(0.5, 3.0, shape_c)
    u = rng.uniform(-0.3, 0.3, shape_n)
    v = rng.uniform(-0.3, 0.3, shape_n)
    if smooth:
        y, x = np.mgrid[0:ny, 0:nx] / max(nx, ny)
        rho = 1.0 + 0.5 * np.sin(6.0 * x + 1.0) * np.cos(5.0 * y) + 0.05 * rho
        yn, xn = np.mgrid[0:ny + 1, 0:nx + 1] / max(nx, ny)
        u = 0.2 * np.sin(4.0 * xn) * np.cos(3.0 * yn) + 0.02 * u
        v = 0.2 * np.cos(4.0 * xn + 0.5) * np.sin(3.0 * yn) + 0.02 * v
    if not wall_velocity:  # reading A16: no flow through the walls
        u[:, 0] = 0.0
        u[:, -1] = 0.0
        v[0, :] = 0.0
        v[-1, :] = 0.0
    return {"density0": np.ascontiguousarray(rho), "energy0": np.ascontiguousarray(e),
            "xvel0": np.ascontiguousarray(u), "yvel0": np.ascontiguousarray(v)}


# Named benchmark / parity configurations (BASELINE.json configs).
CONFIGS = {
    "C1": dict(nx=64, steps=20),      # configs[0] parity vs oracle
    "C2": dict(nx=960, steps=87),     # configs[1] clover_bm_short shape
    "C3": dict(nx=3840, steps=300),   # configs[2] bandwidth-roofline run
    "C4": dict(nx=7680, steps=300),   # configs[3] strong scaling
    "C5": dict(nx=3840, steps=300),   # configs[4] weak scaling, per GPU
}
