"""Thin ctypes binding of libclover.so (include/clover.h).

Argument marshalling only: every step of the CloverLeaf path runs in the
library's sm_100a kernels.  PyTorch supplies the device workspace (one
uint8 tensor), the CUDA stream and, for multi-GPU runs, the process group
used to broadcast the NCCL unique id.  There is no CPU fallback: if the
library cannot be loaded the import of this module's functions raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import build as _build

c_int32 = ctypes.c_int32
c_int64 = ctypes.c_int64
c_double = ctypes.c_double
c_void_p = ctypes.c_void_p
dptr = ctypes.POINTER(c_double)

CLOVER_OK = 0
PROFILE_SLOTS = 15
ERRORS = {-1: "ARG", -2: "CUDA", -3: "NCCL", -4: "WORKSPACE", -5: "SMALL_DT", -6: "NEG_VOLUME",
          -7: "STATE", -8: "NAN"}

FIELDS = {"density0": 0, "energy0": 1, "pressure": 2, "viscosity": 3, "soundspeed": 4,
          "xvel0": 5, "yvel0": 6, "vol_flux_x": 11, "vol_flux_y": 12,
          "mass_flux_x": 13, "mass_flux_y": 14}
GEOM = {"rectangle": 1, "circle": 2, "point": 3}
KIND = {"cell": 0, "xvel": 1, "yvel": 2, "xface": 3, "yface": 4}
# internal buffer ids (csrc/clover_engine.cu enum Buf) for debug reads
BUF = {"d0": 0, "e0": 1, "u0": 2, "v0": 3, "q": 4, "d1": 5, "e1": 6, "u1": 7, "v1": 8,
       "fy": 9, "fx": 10, "d2": 11, "e2": 12, "u2": 13, "v2": 14, "mx": 15,
       "my": 16, "scr": 17}
EXPORTS = ["clover_workspace_bytes", "clover_nccl_unique_id", "clover_init", "clover_step",
           "clover_step_host", "clover_field_summary", "clover_get_clock", "clover_dt_history",
           "clover_read_field", "clover_read_field_window", "clover_write_field", "clover_sync", "clover_set_graphs",
           "clover_kernels_per_step", "clover_launch_count", "clover_local_block", "clover_debug_partial_step", "clover_debug_read_buffer",
           "clover_profile_steps", "clover_profile_name", "clover_debug_div_check",
           "clover_debug_fix_count", "clover_debug_set_fusion", "clover_debug_set_overlap",
           "clover_set_deep_halo", "clover_deep_halo_active",
           "clover_checkpoint_plan", "clover_debug_set_virtual_remote", "clover_checkpoint_bytes", "clover_checkpoint", "clover_restart", "clover_finalize", "clover_error_string", "clover_last_error", "clover_abi_version"]


class CloverGrid(ctypes.Structure):
    _fields_ = [("x_cells", c_int32), ("y_cells", c_int32),
                ("xmin", c_double), ("ymin", c_double), ("xmax", c_double), ("ymax", c_double),
                ("dtinit", c_double), ("dtmax", c_double), ("dtmin", c_double), ("dtrise", c_double),
                ("dtc_safe", c_double), ("dtu_safe", c_double), ("dtv_safe", c_double),
                ("dtdiv_safe", c_double), ("advect_x_first", c_int32), ("face_mirror", c_int32)]


class CloverState(ctypes.Structure):
    _fields_ = [("density", c_double), ("energy", c_double), ("xvel", c_double), ("yvel", c_double),
                ("geometry", c_int32), ("xmin", c_double), ("xmax", c_double), ("ymin", c_double),
                ("ymax", c_double), ("radius", c_double)]


SENDRECV_FN = ctypes.CFUNCTYPE(ctypes.c_int, c_void_p, c_int32, ctypes.POINTER(c_int32),
                               ctypes.POINTER(ctypes.POINTER(c_double)), ctypes.POINTER(c_int64),
                               ctypes.POINTER(ctypes.POINTER(c_double)), ctypes.POINTER(c_int64))
ALLREDUCE_FN = ctypes.CFUNCTYPE(ctypes.c_int, c_void_p, ctypes.POINTER(ctypes.c_uint64))
ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int, c_void_p, ctypes.POINTER(c_double), c_int64,
                                ctypes.POINTER(c_double))


class CloverHostTransport(ctypes.Structure):
    _fields_ = [("user", c_void_p), ("sendrecv", SENDRECV_FN), ("allreduce_min_u64", ALLREDUCE_FN),
                ("allgather_f64", ALLGATHER_FN)]


class CloverDist(ctypes.Structure):
    _fields_ = [("rank", c_int32), ("nranks", c_int32), ("px", c_int32), ("py", c_int32),
                ("nccl_unique_id", c_void_p), ("host_transport", ctypes.POINTER(CloverHostTransport))]


class CloverSummary(ctypes.Structure):
    _fields_ = [("vol", c_double), ("mass", c_double), ("ie", c_double), ("ke", c_double),
                ("press", c_double)]


_lib = None


def lib_path() -> str:
    # CLOVER_LIB: path of an A/B variant of the same library (scripts/ab_variants.py)
    return os.environ.get("CLOVER_LIB", _build.LIB)


def load(build_if_missing: bool = True):
    """Load libclover.so (building it first if missing or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    path = lib_path()
    if build_if_missing and path == _build.LIB:
        _build.build()
    if not os.path.exists(path):
        raise RuntimeError(f"libclover.so not found at {path}; run __graft_entry__.build()")
    L = ctypes.CDLL(path)
    P = ctypes.POINTER
    L.clover_workspace_bytes.argtypes = [P(CloverGrid), P(CloverDist), P(c_int64)]
    L.clover_nccl_unique_id.argtypes = [c_void_p]
    L.clover_init.argtypes = [P(CloverGrid), P(CloverState), c_int32, P(CloverDist), c_void_p,
                              c_int64, c_void_p, P(c_void_p)]
    L.clover_step.argtypes = [c_void_p, c_int32]
    L.clover_step_host.argtypes = [c_void_p, c_int32] + [dptr] * 8
    L.clover_field_summary.argtypes = [c_void_p, P(CloverSummary)]
    L.clover_get_clock.argtypes = [c_void_p, P(c_int32), dptr, dptr]
    L.clover_dt_history.argtypes = [c_void_p, c_int32, c_int32, dptr]
    L.clover_read_field.argtypes = [c_void_p, c_int32, dptr, c_int64]
    L.clover_write_field.argtypes = [c_void_p, c_int32, dptr, c_int64]
    if hasattr(L, "clover_read_field_window"):
        L.clover_read_field_window.argtypes = [c_void_p, c_int32, c_int32, c_int32, c_int32, c_int32,
                                               dptr]
    L.clover_sync.argtypes = [c_void_p]
    L.clover_set_graphs.argtypes = [c_void_p, c_int32]
    L.clover_kernels_per_step.argtypes = [c_void_p, P(c_int32)]
    if hasattr(L, "clover_launch_count"):
        L.clover_launch_count.argtypes = [c_void_p, P(ctypes.c_int64)]
    if hasattr(L, "clover_local_block"):
        L.clover_local_block.argtypes = [c_void_p, P(c_int32)]
    L.clover_debug_partial_step.argtypes = [c_void_p, c_int32]
    L.clover_debug_read_buffer.argtypes = [c_void_p, c_int32, c_int32, dptr, c_int64]
    L.clover_profile_steps.argtypes = [c_void_p, c_int32, dptr, ctypes.POINTER(c_int64), c_int32]
    L.clover_profile_name.argtypes = [c_int32]
    L.clover_profile_name.restype = ctypes.c_char_p
    if hasattr(L, "clover_debug_fix_count"):  # absent from older builds (A/B harness)
        L.clover_debug_fix_count.argtypes = [c_void_p, ctypes.POINTER(c_int64)]
    if hasattr(L, "clover_debug_set_fusion"):
        L.clover_debug_set_fusion.argtypes = [c_void_p, c_int32]
    if hasattr(L, "clover_debug_set_overlap"):
        L.clover_debug_set_overlap.argtypes = [c_void_p, c_int32]
    if hasattr(L, "clover_set_deep_halo"):  # (older A/B builds lack the newer calls)
        L.clover_set_deep_halo.argtypes = [c_void_p, c_int32]
        L.clover_deep_halo_active.argtypes = [c_void_p, P(c_int32)]
    L.clover_debug_div_check.argtypes = [c_int64, ctypes.c_uint64, c_int32, ctypes.POINTER(c_int64), dptr]
    L.clover_checkpoint_plan.argtypes = [c_int32, ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(c_int32),
                                         ctypes.POINTER(ctypes.c_char_p)]
    L.clover_checkpoint_bytes.argtypes = [c_void_p, ctypes.POINTER(c_int64)]
    L.clover_checkpoint.argtypes = [c_void_p, c_void_p, c_int64]
    L.clover_restart.argtypes = [c_void_p, c_void_p, c_int64]
    L.clover_debug_set_virtual_remote.argtypes = [c_void_p, c_int32]
    L.clover_finalize.argtypes = [c_void_p]
    L.clover_error_string.argtypes = [c_int32]
    L.clover_error_string.restype = ctypes.c_char_p
    L.clover_last_error.restype = ctypes.c_char_p
    for name in EXPORTS:
        if os.environ.get("CLOVER_LIB") and not hasattr(L, name):
            continue  # an older build under the A/B harness
        if name not in ("clover_error_string", "clover_last_error", "clover_profile_name"):
            getattr(L, name).restype = c_int32
    _lib = L
    return L


class CloverError(RuntimeError):
    def __init__(self, code, where):
        L = load(False)
        msg = L.clover_last_error().decode(errors="replace")
        super().__init__(f"{where} failed: {ERRORS.get(code, code)} ({msg})")
        self.code = code


def _check(rc, where):
    if rc != CLOVER_OK:
        raise CloverError(rc, where)


def grid_from_deck(deck: dict) -> CloverGrid:
    return CloverGrid(x_cells=deck["x_cells"], y_cells=deck["y_cells"], xmin=deck["xmin"],
                      ymin=deck["ymin"], xmax=deck["xmax"], ymax=deck["ymax"],
                      dtinit=deck.get("initial_timestep", 0.04), dtmax=deck.get("max_timestep", 0.04),
                      dtmin=deck.get("dtmin", 0.0), dtrise=deck.get("timestep_rise", 1.5),
                      dtc_safe=deck.get("dtc_safe", 0.0), dtu_safe=deck.get("dtu_safe", 0.0),
                      dtv_safe=deck.get("dtv_safe", 0.0), dtdiv_safe=deck.get("dtdiv_safe", 0.0),
                      advect_x_first=int(deck.get("advect_x_first", 1)),
                      face_mirror=int(deck.get("face_mirror", 0)))


def states_from_deck(deck: dict):
    sts = deck["states"]
    arr = (CloverState * len(sts))()
    for i, s in enumerate(sts):
        arr[i] = CloverState(density=s["density"], energy=s["energy"], xvel=s.get("xvel", 0.0),
                             yvel=s.get("yvel", 0.0), geometry=GEOM[s.get("geometry", "rectangle")],
                             xmin=s.get("xmin", 0.0), xmax=s.get("xmax", 0.0),
                             ymin=s.get("ymin", 0.0), ymax=s.get("ymax", 0.0),
                             radius=s.get("radius", 0.0))
    return arr


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(load().clover_nccl_unique_id(buf), "clover_nccl_unique_id")
    return buf.raw


def field_shape(name_or_kind: str, nx: int, ny: int):
    k = name_or_kind
    if k in ("xvel0", "yvel0", "xvel", "yvel"):
        return (ny + 1, nx + 1)
    if k in ("vol_flux_x", "mass_flux_x", "xface"):
        return (ny, nx + 1)
    if k in ("vol_flux_y", "mass_flux_y", "yface"):
        return (ny + 1, nx)
    return (ny, nx)


CKPT_DATASETS = ["density0", "energy0", "xvel0", "yvel0", "pressure", "soundspeed", "viscosity",
                 "density1", "energy1", "xvel1", "yvel1", "vol_flux_x", "vol_flux_y",
                 "mass_flux_x", "mass_flux_y"]


def checkpoint_plan(loop: int):
    """(loop name, datasets a checkpoint entered before `loop` must save)."""
    m = ctypes.c_uint32(); n = c_int32(); name = ctypes.c_char_p()
    _check(load().clover_checkpoint_plan(loop, ctypes.byref(m), ctypes.byref(n), ctypes.byref(name)),
           "clover_checkpoint_plan")
    return name.value.decode(), [d for i, d in enumerate(CKPT_DATASETS) if m.value >> i & 1]


def debug_div_check(n: int, seed: int = 1, emax: int = 60):
    """Bitwise check of the library's fp64 division against IEEE a/b."""
    bad = c_int64()
    ex = np.zeros(2, dtype=np.float64)
    _check(load().clover_debug_div_check(n, seed, emax, ctypes.byref(bad), ex.ctypes.data_as(dptr)),
           "clover_debug_div_check")
    return bad.value, (float(ex[0]), float(ex[1]))


class Clover:
    """One CloverLeaf run on the current CUDA device.

    deck: workloads-style dict.  px, py: chunk grid; rank/nranks and
    unique_id for multi-process NCCL runs.  stream: torch.cuda.Stream (or
    None = torch's current stream)."""

    def __init__(self, deck: dict, px: int = 1, py: int = 1, rank: int = 0, nranks: int = 1,
                 unique_id: bytes | None = None, stream=None, device=None, host_transport=None):
        import torch  # device memory + streams only
        L = load()
        self.nx, self.ny = deck["x_cells"], deck["y_cells"]
        self._grid = grid_from_deck(deck)
        self._states = states_from_deck(deck)
        self._uid = ctypes.create_string_buffer(unique_id, 128) if unique_id else None
        # host_transport: an object with the three clover_host_transport
        # collectives (paper_conf_cluster_regulymg15_b200.dist.GlooHostTransport);
        # the ctypes callbacks are kept alive with the context
        self._ht = host_transport.c_struct() if host_transport is not None else None
        self._dist = CloverDist(rank=rank, nranks=nranks, px=px, py=py,
                                nccl_unique_id=ctypes.cast(self._uid, c_void_p) if self._uid else None,
                                host_transport=ctypes.pointer(self._ht) if self._ht is not None else None)
        nbytes = c_int64()
        _check(L.clover_workspace_bytes(ctypes.byref(self._grid), ctypes.byref(self._dist),
                                        ctypes.byref(nbytes)), "clover_workspace_bytes")
        dev = torch.device("cuda", torch.cuda.current_device()) if device is None else device
        self.workspace = torch.empty(nbytes.value + 256, dtype=torch.uint8, device=dev)
        base = self.workspace.data_ptr()
        aligned = (base + 255) // 256 * 256
        self.stream = stream if stream is not None else torch.cuda.current_stream(dev)
        self._ctx = c_void_p()
        _check(L.clover_init(ctypes.byref(self._grid), self._states, len(self._states),
                             ctypes.byref(self._dist), c_void_p(aligned), nbytes.value,
                             c_void_p(self.stream.cuda_stream), ctypes.byref(self._ctx)),
               "clover_init")

    # -- API mirrors include/clover.h --------------------------------------
    def step(self, n: int = 1):
        _check(load().clover_step(self._ctx, n), "clover_step")

    def step_host(self, n, fields_in: dict, fields_out: dict):
        args = []
        for name in ("density0", "energy0", "xvel0", "yvel0"):
            a = fields_in.get(name)
            args.append(a.ctypes.data_as(dptr) if a is not None else None)
        for name in ("density0", "energy0", "xvel0", "yvel0"):
            a = fields_out.get(name)
            args.append(a.ctypes.data_as(dptr) if a is not None else None)
        _check(load().clover_step_host(self._ctx, n, *args), "clover_step_host")

    def sync(self):
        _check(load().clover_sync(self._ctx), "clover_sync")

    def set_graphs(self, on: bool):
        _check(load().clover_set_graphs(self._ctx, 1 if on else 0), "clover_set_graphs")

    def kernels_per_step(self) -> int:
        n = c_int32()
        _check(load().clover_kernels_per_step(self._ctx, ctypes.byref(n)), "clover_kernels_per_step")
        return n.value

    def local_block(self):
        """(j0, k0, width, height): this process's chunks in global cells."""
        a = (c_int32 * 4)()
        _check(load().clover_local_block(self._ctx, a), "clover_local_block")
        return tuple(a)

    def launch_count(self) -> int:
        """Step kernels launched on this context so far (clover_launch_count)."""
        n = ctypes.c_int64()
        _check(load().clover_launch_count(self._ctx, ctypes.byref(n)), "clover_launch_count")
        return n.value

    def field_summary(self) -> dict:
        s = CloverSummary()
        _check(load().clover_field_summary(self._ctx, ctypes.byref(s)), "clover_field_summary")
        return dict(vol=s.vol, mass=s.mass, ie=s.ie, ke=s.ke, press=s.press)

    def clock(self) -> dict:
        st = c_int32(); t = c_double(); dt = c_double()
        _check(load().clover_get_clock(self._ctx, ctypes.byref(st), ctypes.byref(t), ctypes.byref(dt)),
               "clover_get_clock")
        return dict(step=st.value, time=t.value, dt=dt.value)

    def dt_history(self, first: int, n: int) -> np.ndarray:
        out = np.zeros(n, dtype=np.float64)
        _check(load().clover_dt_history(self._ctx, first, n, out.ctypes.data_as(dptr)), "clover_dt_history")
        return out

    def read(self, name: str) -> np.ndarray:
        a = np.zeros(field_shape(name, self.nx, self.ny), dtype=np.float64)
        _check(load().clover_read_field(self._ctx, FIELDS[name], a.ctypes.data_as(dptr), a.size),
               f"clover_read_field({name})")
        return a

    def read_window(self, name: str, j0: int, k0: int, w: int, h: int) -> np.ndarray:
        """Rows k0..k0+h-1, columns j0..j0+w-1 (global, 1-based) of a field."""
        a = np.zeros((h, w), dtype=np.float64)
        _check(load().clover_read_field_window(self._ctx, FIELDS[name], j0, k0, w, h,
                                               a.ctypes.data_as(dptr)),
               f"clover_read_field_window({name})")
        return a

    def write(self, name: str, a: np.ndarray):
        a = np.ascontiguousarray(a, dtype=np.float64)
        assert a.shape == field_shape(name, self.nx, self.ny), (name, a.shape)
        _check(load().clover_write_field(self._ctx, FIELDS[name], a.ctypes.data_as(dptr), a.size),
               f"clover_write_field({name})")

    def load_state(self, fields: dict):
        for k, v in fields.items():
            self.write(k, v)

    def profile_steps(self, n: int) -> dict:
        """Per-kernel-type summed CUDA-event durations over n steps (direct
        launches, event after every kernel on the work stream)."""
        L = load()
        ms = np.zeros(PROFILE_SLOTS, dtype=np.float64)
        cnt = np.zeros(PROFILE_SLOTS, dtype=np.int64)
        _check(L.clover_profile_steps(self._ctx, n, ms.ctypes.data_as(dptr),
                                      cnt.ctypes.data_as(ctypes.POINTER(c_int64)), PROFILE_SLOTS),
               "clover_profile_steps")
        return {L.clover_profile_name(i).decode(): (float(ms[i]), int(cnt[i]))
                for i in range(PROFILE_SLOTS) if cnt[i]}

    def checkpoint(self) -> bytes:
        n = c_int64()
        _check(load().clover_checkpoint_bytes(self._ctx, ctypes.byref(n)), "clover_checkpoint_bytes")
        buf = ctypes.create_string_buffer(n.value)
        _check(load().clover_checkpoint(self._ctx, buf, n.value), "clover_checkpoint")
        return buf.raw

    def restart(self, blob: bytes):
        buf = ctypes.create_string_buffer(blob, len(blob))
        _check(load().clover_restart(self._ctx, buf, len(blob)), "clover_restart")

    def debug_set_virtual_remote(self, on, nccl: bool = False, lsa: bool = False):
        """on: chunk boundaries through the remote (pack/staging/unpack) path;
        nccl: the messages through a one-rank NCCL communicator (send/recv to
        self) and dt through a one-rank NCCL all-reduce; lsa: the messages
        as device-initiated stores into a one-rank NCCL symmetric window
        (LSA barriers), dt as with nccl."""
        mode = (3 if lsa else 2 if nccl else 1) if on else 0
        _check(load().clover_debug_set_virtual_remote(self._ctx, mode), "clover_debug_set_virtual_remote")

    def debug_partial_step(self, nkernels: int):
        _check(load().clover_debug_partial_step(self._ctx, nkernels), "clover_debug_partial_step")

    def debug_set_fusion(self, enable, walls_only: bool = False):
        """Fused sweeps on (default), off (separate cell / momentum kernels),
        or with walls_only the fused y sweep only where every chunk has both
        y walls (round-1 behaviour: separate y kernels at y chunk boundaries)."""
        v = (2 if walls_only else 1) if enable else 0
        _check(load().clover_debug_set_fusion(self._ctx, v), "clover_debug_set_fusion")

    def debug_set_overlap(self, enable: bool):
        """Boundary segments first + the exchange overlapped with the interior
        (y strips with remote / virtual-remote exchanges; default off)."""
        _check(load().clover_debug_set_overlap(self._ctx, 1 if enable else 0), "clover_debug_set_overlap")

    def set_deep_halo(self, enable: bool):
        """Deep halos (one 7-row state exchange per step on y-strip layouts;
        include/clover.h clover_set_deep_halo)."""
        _check(load().clover_set_deep_halo(self._ctx, 1 if enable else 0), "clover_set_deep_halo")

    def deep_halo_active(self) -> bool:
        n = c_int32()
        _check(load().clover_deep_halo_active(self._ctx, ctypes.byref(n)), "clover_deep_halo_active")
        return bool(n.value)

    def debug_fix_count(self) -> int:
        """Warp segments recomputed so far by the IEEE-division fixup launches."""
        n = c_int64()
        _check(load().clover_debug_fix_count(self._ctx, ctypes.byref(n)), "clover_debug_fix_count")
        return n.value

    def debug_read(self, buf: str, kind: str) -> np.ndarray:
        a = np.zeros(field_shape(kind, self.nx, self.ny), dtype=np.float64)
        _check(load().clover_debug_read_buffer(self._ctx, BUF[buf], KIND[kind], a.ctypes.data_as(dptr), a.size),
               "clover_debug_read_buffer")
        return a

    def close(self):
        if getattr(self, "_ctx", None) is not None and self._ctx.value:
            rc = load().clover_finalize(self._ctx)
            self._ctx = c_void_p()
            _check(rc, "clover_finalize")

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
