"""CPU checks of the C-ABI boundary (no GPU): the library builds for
sm_100a, loads, exports every function include/clover.h declares, rejects
bad arguments before touching the device, and ships real sm_100a SASS."""
from __future__ import annotations

import ctypes
import os
import re
import subprocess

from paper_conf_cluster_regulymg15_b200 import clover as cb

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    src = open(os.path.join(ROOT, "include", "clover.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(clover_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_north_star_entry_points():
    names = declared_functions()
    for n in ("clover_init", "clover_step", "clover_field_summary", "clover_finalize"):
        assert n in names


def test_library_exports_every_declared_symbol():
    L = cb.load()
    missing = [n for n in declared_functions() if not hasattr(L, n)]
    assert not missing, missing
    assert set(declared_functions()) <= set(cb.EXPORTS)
    assert L.clover_abi_version() == 2


def test_error_strings_and_validation_without_gpu():
    L = cb.load()
    assert L.clover_error_string(-5) == b"small timestep (dt < dtmin)"
    from workloads import bm_deck
    g = cb.grid_from_deck(bm_deck(64))
    nb = ctypes.c_int64()
    assert L.clover_workspace_bytes(ctypes.byref(g), None, ctypes.byref(nb)) == 0
    assert nb.value > 18 * 64 * 64 * 8
    bad = cb.grid_from_deck(bm_deck(3))
    assert L.clover_workspace_bytes(ctypes.byref(bad), None, ctypes.byref(nb)) == -1
    assert b">= 4" in L.clover_last_error()
    d = cb.CloverDist(rank=0, nranks=3, px=2, py=1, nccl_unique_id=None)
    assert L.clover_workspace_bytes(ctypes.byref(g), ctypes.byref(d), ctypes.byref(nb)) == -1
    # init with a NULL workspace is refused before any CUDA call
    ctx = ctypes.c_void_p()
    st = cb.states_from_deck(bm_deck(64))
    rc = L.clover_init(ctypes.byref(g), st, len(st), None, None, 0, None, ctypes.byref(ctx))
    assert rc == -4 and not ctx.value


def test_decomposed_workspace_covers_all_chunks():
    L = cb.load()
    from workloads import bm_deck
    g = cb.grid_from_deck(bm_deck(128))
    one = ctypes.c_int64(); four = ctypes.c_int64()
    assert L.clover_workspace_bytes(ctypes.byref(g), None, ctypes.byref(one)) == 0
    d = cb.CloverDist(rank=0, nranks=1, px=2, py=2, nccl_unique_id=None)
    assert L.clover_workspace_bytes(ctypes.byref(g), ctypes.byref(d), ctypes.byref(four)) == 0
    assert four.value > one.value
    d2 = cb.CloverDist(rank=1, nranks=4, px=2, py=2, nccl_unique_id=None)
    assert L.clover_workspace_bytes(ctypes.byref(g), ctypes.byref(d2), ctypes.byref(one)) == -1  # no uid


def test_sass_is_sm100a_and_has_no_cpu_fallback():
    lib = cb.lib_path()
    out = subprocess.run(["cuobjdump", "--list-elf", lib], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
    for k in ("ks_visc_dt", "ks_lagrangian", "ks_advec_cell_x", "ks_advec_mom_y", "k_dt_finalize"):
        assert k in sass
    # the Lagrangian kernel stages rows with TMA tensor copies (3D: row x field)
    lag = sass[sass.index("Function : _ZN6clover13ks_lagrangian"):]
    lag = lag[:lag.index("Function :", 10)] if "Function :" in lag[10:] else lag
    assert "UTMALDG.3D" in lag and "SYNCS" in lag


def test_product_package_does_not_touch_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_cluster_regulymg15_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dp, f)).read()
                for bad in ("import oracle", "from oracle", "clover_oracle", "liboracle",
                            "oracle_"):
                    assert bad not in txt, (f, bad)
