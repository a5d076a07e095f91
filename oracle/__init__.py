"""ctypes wrapper of the CPU ORACLE (clover_oracle.cpp).

TEST INFRASTRUCTURE ONLY: tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this; the product package
(paper_conf_cluster_regulymg15_b200) never does.

The oracle follows SURVEY.md 8(c) (CloverLeaf 2D reference kernels; the
method is named in PAPER.md:209 sec. V).  See clover_oracle.cpp for the
per-function citations and DESIGN.md for the pins.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")

FIELDS = {
    "density0": 0, "energy0": 1, "pressure": 2, "viscosity": 3, "soundspeed": 4,
    "xvel0": 5, "yvel0": 6, "density1": 7, "energy1": 8, "xvel1": 9, "yvel1": 10,
    "vol_flux_x": 11, "vol_flux_y": 12, "mass_flux_x": 13, "mass_flux_y": 14,
}
STAGES = {"timestep": 0, "pdv_predict": 1, "accelerate": 2, "pdv_correct": 3,
          "flux_calc": 4, "advection": 5, "reset": 6,
          "adv_cell1": 7, "adv_mom1": 8, "adv_cell2": 9, "adv_mom2": 10}
GEOM = {"rectangle": 1, "circle": 2, "point": 3}


class OracleGrid(ctypes.Structure):
    _fields_ = [("x_cells", ctypes.c_int32), ("y_cells", ctypes.c_int32),
                ("xmin", ctypes.c_double), ("ymin", ctypes.c_double),
                ("xmax", ctypes.c_double), ("ymax", ctypes.c_double),
                ("dtinit", ctypes.c_double), ("dtmax", ctypes.c_double),
                ("dtmin", ctypes.c_double), ("dtrise", ctypes.c_double),
                ("dtc_safe", ctypes.c_double), ("dtu_safe", ctypes.c_double),
                ("dtv_safe", ctypes.c_double), ("dtdiv_safe", ctypes.c_double),
                ("advect_x_first", ctypes.c_int32), ("face_mirror", ctypes.c_int32)]


class OracleState(ctypes.Structure):
    _fields_ = [("density", ctypes.c_double), ("energy", ctypes.c_double),
                ("xvel", ctypes.c_double), ("yvel", ctypes.c_double),
                ("geometry", ctypes.c_int32),
                ("xmin", ctypes.c_double), ("xmax", ctypes.c_double),
                ("ymin", ctypes.c_double), ("ymax", ctypes.c_double),
                ("radius", ctypes.c_double)]


CLI_PATH = os.path.join(_HERE, "clover_oracle")  # c.15 command-line driver


def build(force: bool = False) -> str:
    srcs = [os.path.join(_HERE, f) for f in ("clover_oracle.cpp", "clover_oracle.h",
                                             "clover_oracle_main.cpp")]
    newest = max(os.path.getmtime(s) for s in srcs)
    for target in (_LIB_PATH, CLI_PATH):
        if force or not os.path.exists(target) or os.path.getmtime(target) < newest:
            if force:
                subprocess.check_call(["make", "-s", "-B", "-C", _HERE, os.path.basename(target)])
            else:
                subprocess.check_call(["make", "-s", "-C", _HERE, os.path.basename(target)])
    return _LIB_PATH


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        vp = ctypes.c_void_p
        dp = ctypes.POINTER(ctypes.c_double)
        L.oracle_create.restype = vp
        L.oracle_create.argtypes = [ctypes.POINTER(OracleGrid), ctypes.POINTER(OracleState), ctypes.c_int32]
        L.oracle_destroy.argtypes = [vp]
        L.oracle_step.restype = ctypes.c_int32
        L.oracle_step.argtypes = [vp, ctypes.c_int32, dp]
        L.oracle_run_stage.restype = ctypes.c_int32
        L.oracle_run_stage.argtypes = [vp, ctypes.c_int32]
        L.oracle_field_summary.argtypes = [vp, dp]
        L.oracle_field_summary_compensated.argtypes = [vp, dp]
        L.oracle_clock.argtypes = [vp, ctypes.POINTER(ctypes.c_int32), dp, dp, dp]
        L.oracle_read_field.restype = ctypes.c_int32
        L.oracle_read_field.argtypes = [vp, ctypes.c_int32, dp, ctypes.c_int64]
        L.oracle_write_field.restype = ctypes.c_int32
        L.oracle_write_field.argtypes = [vp, ctypes.c_int32, dp, ctypes.c_int64]
        L.oracle_refresh.argtypes = [vp]
        _lib = L
    return _lib


def field_shape(name: str, nx: int, ny: int):
    if name in ("xvel0", "yvel0", "xvel1", "yvel1"):
        return (ny + 1, nx + 1)
    if name in ("vol_flux_x", "mass_flux_x"):
        return (ny, nx + 1)
    if name in ("vol_flux_y", "mass_flux_y"):
        return (ny + 1, nx)
    return (ny, nx)


class Oracle:
    """One oracle instance = one CloverLeaf chunk covering the whole mesh."""

    def __init__(self, deck: dict):
        g = OracleGrid(x_cells=deck["x_cells"], y_cells=deck["y_cells"],
                       xmin=deck["xmin"], ymin=deck["ymin"], xmax=deck["xmax"], ymax=deck["ymax"],
                       dtinit=deck.get("initial_timestep", 0.04), dtmax=deck.get("max_timestep", 0.04),
                       dtmin=deck.get("dtmin", 0.0), dtrise=deck.get("timestep_rise", 1.5),
                       dtc_safe=deck.get("dtc_safe", 0.0), dtu_safe=deck.get("dtu_safe", 0.0),
                       dtv_safe=deck.get("dtv_safe", 0.0), dtdiv_safe=deck.get("dtdiv_safe", 0.0),
                       advect_x_first=int(deck.get("advect_x_first", 1)),
                       face_mirror=int(deck.get("face_mirror", 0)))
        sts = deck["states"]
        arr = (OracleState * len(sts))()
        for i, s in enumerate(sts):
            arr[i] = OracleState(density=s["density"], energy=s["energy"], xvel=s.get("xvel", 0.0),
                                 yvel=s.get("yvel", 0.0), geometry=GEOM[s.get("geometry", "rectangle")],
                                 xmin=s.get("xmin", 0.0), xmax=s.get("xmax", 0.0),
                                 ymin=s.get("ymin", 0.0), ymax=s.get("ymax", 0.0),
                                 radius=s.get("radius", 0.0))
        self.nx, self.ny = deck["x_cells"], deck["y_cells"]
        self._c = lib().oracle_create(ctypes.byref(g), arr, len(sts))
        if not self._c:
            raise ValueError("oracle_create rejected the deck")

    def close(self):
        if self._c:
            lib().oracle_destroy(self._c)
            self._c = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def step(self, n: int = 1) -> np.ndarray:
        dts = np.zeros(max(n, 1), dtype=np.float64)
        rc = lib().oracle_step(self._c, n, dts.ctypes.data_as(ctypes.POINTER(ctypes.c_double)))
        if rc != 0:
            raise RuntimeError(f"oracle_step failed rc={rc}")
        return dts[:n]

    def run_stage(self, name: str) -> int:
        return lib().oracle_run_stage(self._c, STAGES[name])

    def field_summary(self, compensated: bool = False) -> dict:
        out = np.zeros(5, dtype=np.float64)
        f = lib().oracle_field_summary_compensated if compensated else lib().oracle_field_summary
        f(self._c, out.ctypes.data_as(ctypes.POINTER(ctypes.c_double)))
        return dict(zip(("vol", "mass", "ie", "ke", "press"), out.tolist()))

    def clock(self):
        s = ctypes.c_int32(); t = ctypes.c_double(); dt = ctypes.c_double(); dto = ctypes.c_double()
        lib().oracle_clock(self._c, ctypes.byref(s), ctypes.byref(t), ctypes.byref(dt), ctypes.byref(dto))
        return dict(step=s.value, time=t.value, dt=dt.value, dtold=dto.value)

    def read(self, name: str) -> np.ndarray:
        a = np.zeros(field_shape(name, self.nx, self.ny), dtype=np.float64)
        rc = lib().oracle_read_field(self._c, FIELDS[name], a.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), a.size)
        if rc:
            raise ValueError(name)
        return a

    def write(self, name: str, a: np.ndarray):
        a = np.ascontiguousarray(a, dtype=np.float64)
        assert a.shape == field_shape(name, self.nx, self.ny), (name, a.shape)
        rc = lib().oracle_write_field(self._c, FIELDS[name], a.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), a.size)
        if rc:
            raise ValueError(name)

    def refresh(self):
        lib().oracle_refresh(self._c)

    def load_state(self, fields: dict):
        """Overwrite density0/energy0/xvel0/yvel0 interiors, then redo the
        start-of-run EOS + halo update (start.f90 tail)."""
        for k, v in fields.items():
            self.write(k, v)
        self.refresh()
