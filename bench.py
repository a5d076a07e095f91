#!/usr/bin/env python
"""Benchmark of the B200-native CloverLeaf 2D timestep (BASELINE.json).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl clover|reference]

One bench "step" = one full CloverLeaf timestep (every SURVEY 8(a) row:
EOS, viscosity, calc_dt + min-reduction, PdV predictor/corrector,
accelerate, flux_calc, both advection sweeps, reset, halo updates).

N=1 workload: BASELINE configs[2], the bm deck on 3840x3840 cells (the
"1 GPU bandwidth-roofline run"; configs[1] 960^2 and configs[0] 64^2 are
parity-test cases in tests/).  N>1: configs[4], weak scaling with 3840^2
cells per GPU (reading A4: 2 -> 7680x3840, 4 -> 7680^2, 8 -> 15360x7680, all
on [0,10]^2, y-strip chunks), one process per GPU, NCCL halo exchange and dt
MIN all-reduce; --strong: configs[3], 7680^2 over the ranks.

Prints ONE JSON line (rank 0).  --impl reference times the CPU oracle (the
reference arm of this tier) on the host cores.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "cell-updates/sec per step and achieved HBM GB/s vs peak, at 1/2/4/8 B200"
UNIT = "cell-updates/s"

# Algorithmic HBM bytes per cell per launch: fp64
# words each kernel must read + write once (8 B each).
ALGO_BYTES_PER_CELL = {
    "k_visc_dt": 8 * (4 + 1),            # rho0 e0 u0 v0 -> q
    "k_dt_finalize": 0,
    "k_lagrangian": 8 * (5 + 6),         # rho0 e0 q u0 v0 -> rho1 e1 u1 v1 Fx Fy
    "k_advec_cell_x<1>": 8 * (4 + 3),    # rho e Fx Fy -> rho' e' Mx
    "k_advec_cell_y<1>": 8 * (4 + 3),
    "k_advec_cell_x<2>": 8 * (3 + 3),    # rho e Fx -> rho e Mx
    "k_advec_cell_y<2>": 8 * (3 + 3),
    "k_advec_mom_x<1>": 8 * (5 + 2),     # rho M Fy u v -> u v
    "k_advec_mom_y<1>": 8 * (5 + 2),
    "k_advec_mom_x<2>": 8 * (4 + 2),     # rho M u v -> u v
    "k_advec_mom_y<2>": 8 * (4 + 2),
    "k_advec_x<1>": 8 * (6 + 4),         # fused x sweep: rho e Fx Fy u v -> rho' e' u v
    "k_advec_x<2>": 8 * (5 + 4),         # rho e Fx u v -> rho' e' u v
    "k_advec_y<1>": 8 * (6 + 4),         # fused y sweep: rho e Fx Fy u v -> rho' e' u v
    "k_advec_y<2>": 8 * (5 + 4),         # rho e Fy u v -> rho' e' u v
}
# (the step total is summed over the kernels actually launched in the
# profile pass below: 280 B/cell-step with the fused sweeps)

# Issue roofline: every SM sub-partition issues at most one
# warp instruction per cycle, 4 per SM.
ISSUE_PER_SM_PER_CLK = 4


def env_int(name, default):
    try:
        return int(os.environ.get(name, default))
    except ValueError:
        return default


# BASELINE.json north_star: "achieved HBM GB/s against about 8 TB/s per B200"
NOMINAL_HBM_GBS = 8000.0


def ncu_window(cx, cy):
    """S:8(d) hbm_gbs from the committed ncu capture (profiles/ncu_traffic.json,
    written by scripts/summarize_profiles.py): the sum of DRAM bytes over the
    sum of kernel time of the captured window's streaming kernels, when the
    capture's mesh is this rank's chunk."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as fh:
            tr = json.load(fh)
        w = tr.get("window")
        if not w or tuple(tr.get("mesh", [])) != (cx, cy) or not w.get("hbm_gbs"):
            return None
        return {"hbm_gbs": w["hbm_gbs"], "launches": w["launches"], "source": tr.get("source"),
                "how": "sum of ncu dram__bytes (read+write) / sum of gpu__time_duration, "
                       "streaming kernels of the captured steps (cold-cache, serialised launches)"}
    except (OSError, ValueError, KeyError):
        return None


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as fh:
            d = json.load(fh)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.rows = []
        self._stop = threading.Event()
        self._t = None
        self._nv = self._nvml_handle()  # NVML init (~tens of ms) before the timed region

    def _nvml_handle(self):
        """NVML handle of the CUDA device (by UUID, else by index), or None."""
        try:
            import pynvml
            import torch
            pynvml.nvmlInit()
            try:
                u = str(torch.cuda.get_device_properties(self.idx).uuid)
                return pynvml, pynvml.nvmlDeviceGetHandleByUUID(u if u.startswith("GPU-") else "GPU-" + u)
            except Exception:
                return pynvml, pynvml.nvmlDeviceGetHandleByIndex(self.idx)
        except Exception:
            return None

    def _run(self):
        nv = self._nv
        if nv is not None:
            # NVML directly: ~1 ms per sample, so a timed region of tens of
            # milliseconds still gets many samples (nvidia-smi takes ~0.1 s)
            p, h = nv
            bits = (p.nvmlClocksThrottleReasonHwSlowdown, p.nvmlClocksThrottleReasonHwThermalSlowdown,
                    p.nvmlClocksThrottleReasonSwThermalSlowdown, p.nvmlClocksThrottleReasonSwPowerCap)
            while not self._stop.is_set():
                try:
                    sm = p.nvmlDeviceGetClockInfo(h, p.NVML_CLOCK_SM)
                    smax = p.nvmlDeviceGetMaxClockInfo(h, p.NVML_CLOCK_SM)
                    r = p.nvmlDeviceGetCurrentClocksThrottleReasons(h)
                    self.rows.append([str(self.idx), str(sm), str(smax), "", ""] +
                                     ["Active" if r & b else "Not Active" for b in bits])
                except Exception:
                    break
                self._stop.wait(0.001)
            if self.rows:
                return
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True,
                                     text=True, timeout=5).stdout.strip()
                if out:
                    self.rows.append([x.strip() for x in out.split(",")])
            except Exception:
                pass
            self._stop.wait(0.2)

    def start(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()

    def stop(self):
        self._stop.set()
        if self._t:
            self._t.join(timeout=6)
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        smax = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for n, v in zip(names, r[5:9]):
                if v.strip().lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(self.rows),
                "source": "nvml" if self.rows and self.rows[0][3] == "" else "nvidia-smi"}


# The paper's own CloverLeaf numbers (PAPER.md:177-205 Fig. 5, :209, :259
# Fig. 6): context only -- whole-application runtimes whose
# mesh, step count and single-node hardware the paper does not state.
PAPER_CONTEXT = {
    "fig5_runtime_s": {"CUDA original": 14.14, "CUDA OPS": 15.01, "OpenCL GPU original": 16.19,
                       "OpenCL GPU OPS": 16.27, "OpenACC original": 21.67, "OpenACC OPS": 19.82,
                       "32 MPI CPU original": 44.60, "32 MPI CPU OPS": 45.55},
    "fig5_hardware": "not stated (the paper's other single-node runs: Xeon E5-2697 v2 + Tesla K40, "
                     "PAPER.md:93,109); workload not stated",
    "fig6": "ORNL Titan (Cray XK7, K20X GPUs): weak scaling -6% from 1 to 8192 GPUs, -1% from 16 to "
            "65k CPU cores; GPU strong scaling 'does not strong scale very well' (PAPER.md:259)",
    "note": "context only, not a target: no cell-updates/s or GB/s are published (BASELINE.json "
            "published = {})",
}


def host_cpu():
    """CPU model and logical core count of this host (for cpu_baseline)."""
    model = None
    try:
        with open("/proc/cpuinfo") as fh:
            for line in fh:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    sockets = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=5).stdout
        for line in out.splitlines():
            if line.startswith("Socket(s):"):
                sockets = int(line.split(":", 1)[1])
    except Exception:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count(), "sockets": sockets}


def issue_roofline(kernels, top, sm_mhz, nsm):
    """Second roofline: warp instructions per
    launch of the dominant kernel (ncu, profiles/ncu_instr.json, same mesh)
    over its live CUDA-event duration, against the issue peak of nsm SMs x
    4 sub-partitions x 1 warp instruction per cycle at the SM clock sampled
    during the timed region; plus the kernel's fp64-pipe utilisation from the
    same capture."""
    p = os.path.join(ROOT, "profiles", "ncu_instr.json")
    if not os.path.exists(p) or not sm_mhz:
        return None
    with open(p) as fh:
        d = json.load(fh)
    ent = d.get("kernels", {}).get(top)
    if not ent:
        return None
    avg_s = kernels[top]["avg_ms"] / 1e3
    ach = ent["warp_inst_per_launch"] / avg_s / 1e12
    peak = nsm * ISSUE_PER_SM_PER_CLK * sm_mhz * 1e6 / 1e12
    return {"bound": "issue", "kernel": top, "achieved": ach, "peak": peak, "unit": "T warp-inst/s",
            "frac": ach / peak, "thread_inst_per_cell": ent.get("thread_inst_per_cell"),
            "fp64_pipe_pct_active": ent.get("fp64_pipe_pct"),
            "issue_active_pct_ncu": ent.get("issue_active_pct"),
            "peak_source": f"{nsm} SMs x {ISSUE_PER_SM_PER_CLK} warp-inst/clk x median SM clock "
                           f"{sm_mhz:.0f} MHz under load (B200_PROFILING.md unit counts)",
            "inst_source": d.get("source")}


def oracle_rate(deck, steps, warmup=0):
    """Time the CPU oracle (as it stands, single-threaded) on `deck`."""
    from oracle import Oracle
    o = Oracle(deck)
    if warmup:
        o.step(warmup)
    t0 = time.perf_counter()
    o.step(steps)
    t = time.perf_counter() - t0
    o.close()
    cells = deck["x_cells"] * deck["y_cells"]
    return cells * steps / t, t


def arm_mesh(args, world):
    """Global mesh and chunk grid of this run: configs[2] at N = 1,
    configs[4]'s weak series (reading A4) or with --strong configs[3] at N > 1,
    or --mesh."""
    from paper_conf_cluster_regulymg15_b200 import dist as cdist
    if args.strong:
        nx, ny = 7680, 7680
        px, py = cdist.chunk_grid(world, nx, ny)
    else:
        nx, ny, px, py = cdist.weak_mesh(world)
    if args.mesh:
        nx, ny = args.mesh
        px, py = cdist.chunk_grid(world, nx, ny)
    return nx, ny, px, py


def band_deck(nx=3840, ny=3840, rows=240):
    """Bounded sample of the nx x ny bm workload on [0,10]^2: its bottom
    `rows` rows at the same cell size (domain [0,10] x [0, 10*rows/ny])."""
    from workloads import bm_deck
    d = bm_deck(nx, rows)
    d["ymax"] = 10.0 * rows / ny
    return d


def run_reference(args):
    rank = env_int("RANK", 0)
    if rank != 0:
        return
    # the arm's own workload (the same mesh and cell size as `bench.py
    # --gpus N` with these flags), a band of about 0.9 M cells per step
    nx, ny, _, _ = arm_mesh(args, max(args.gpus, env_int("WORLD_SIZE", 1)))
    rows = max(16, min(240, 921600 // nx))
    deck = band_deck(nx, ny, rows)
    from oracle import Oracle
    o = Oracle(deck)
    o.step(args.warmup)
    t0 = time.perf_counter()
    o.step(args.steps)
    t = time.perf_counter() - t0
    cells = deck["x_cells"] * deck["y_cells"]
    v = cells * args.steps / t
    hc = host_cpu()
    sample = (f"oracle (single-threaded C++ -O2) on a bounded sample of the arm's workload: the "
              f"bottom {deck['y_cells']} rows of the {nx}x{ny} bm mesh at the same cell size "
              f"({cells} cells) per step, {args.steps} timed steps after {args.warmup} warm-up")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT,
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1000.0 * t / max(args.steps, 1), "higher_is_better": True,
            "scaling": "strong" if args.strong else "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": f"sample of the {nx}x{ny} CloverLeaf 2D bm deck: "
                                   f"{nx} x {deck['y_cells']} band",
                       "mesh": [deck["x_cells"], deck["y_cells"]], "full_mesh": [nx, ny]},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                             **hc},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="clover", choices=["clover", "reference"])
    ap.add_argument("--mesh", type=int, nargs=2, default=None, help="override global mesh (nx ny)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-full", action="store_true", help="skip the full 300-step configs[2] run")
    ap.add_argument("--no-active", action="store_true",
                    help="skip the fully-active-flow side measurement")
    ap.add_argument("--strong", action="store_true",
                    help="configs[3]: 7680^2 strong-scaled over the ranks (default: configs[4] weak)")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "host"],
                    help="host: gloo host transport, ranks may share a GPU (validates the "
                         "multi-rank path on a one-GPU box; its timing is not a bench value)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
        return

    import numpy as np
    import torch
    import torch.distributed as dist

    rank, world, local = env_int("RANK", 0), env_int("WORLD_SIZE", 1), env_int("LOCAL_RANK", 0)
    if world != args.gpus:
        args.gpus = world
    host_tp = args.transport == "host"
    if host_tp:
        local = local % max(torch.cuda.device_count(), 1)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    from paper_conf_cluster_regulymg15_b200 import Clover, nccl_unique_id
    from paper_conf_cluster_regulymg15_b200 import dist as cdist
    from workloads import bm_deck

    if world > 1:
        if host_tp:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    nx, ny, px, py = arm_mesh(args, world)
    # the bm deck on [0,10]^2 for every mesh (reading A4: the weak-scaling
    # series grows the mesh in both axes on the fixed domain)
    deck = bm_deck(nx, ny, end_step=args.steps)
    uid = cdist.share_unique_id(nccl_unique_id) if world > 1 and not host_tp else None
    ht = cdist.GlooHostTransport() if world > 1 and host_tp else None
    stream = torch.cuda.Stream(dev)
    sim = Clover(deck, px=px, py=py, rank=rank, nranks=world, unique_id=uid, stream=stream,
                 host_transport=ht)
    cells = nx * ny

    # warm-up (also builds the CUDA graphs)
    sim.step(args.warmup)
    sim.sync()
    clocks = ClockSampler(local)
    clocks.start()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    nl0 = sim.launch_count()
    e0.record(stream)
    sim.step(args.steps)
    e1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms = e0.elapsed_time(e1)
    clk = clocks.stop()
    sim.sync()
    ms = cdist.max_over_ranks(ms, None if host_tp else dev)
    value = cells * args.steps / (ms / 1000.0)
    launches = sim.launch_count() - nl0  # counted by the engine, graph launches included
    deep_halo = sim.deep_halo_active()

    # per-kernel CUDA-event durations over a second pass of K steps on the
    # same stream (direct launches, event after every kernel)
    prof = sim.profile_steps(args.steps)
    local_cells = cells // world
    kernels = {}
    for name, (kms, n) in prof.items():
        avg = kms / n
        bpc = ALGO_BYTES_PER_CELL.get(name, 0)
        kernels[name] = {"avg_ms": avg, "launches": n, "share": None,
                         "algo_bytes_per_launch": bpc * local_cells,
                         "achieved_gbs": (bpc * local_cells / (avg / 1e3) / 1e9) if avg > 0 and bpc else None}
    tot = sum(v["avg_ms"] * v["launches"] for v in kernels.values())
    for v in kernels.values():
        v["share"] = v["avg_ms"] * v["launches"] / tot if tot else None
    top = max((k for k in kernels if ALGO_BYTES_PER_CELL.get(k)), key=lambda k: kernels[k]["avg_ms"] * kernels[k]["launches"])
    peak, peak_src = measured_peaks()
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):
        try:
            with open(tp) as fh:
                tr = json.load(fh)
            ent = tr.get("kernels", {}).get(top)
            if ent and tuple(tr.get("mesh", [])) == (nx // px, ny // py):
                traffic = ent["dram_bytes_per_launch"]
        except Exception:
            traffic = None
    ach = kernels[top]["achieved_gbs"]
    step_bpc = sum(ALGO_BYTES_PER_CELL.get(k, 0) * v["launches"] for k, v in kernels.items()) / args.steps
    step_gbs = step_bpc * local_cells * args.steps / (ms / 1e3) / 1e9
    roofline = {"bound": "hbm", "kernel": top, "achieved": ach, "peak": peak, "unit": "GB/s",
                "frac": ach / peak if ach else None, "traffic": traffic, "peak_source": peak_src,
                "step_achieved": step_gbs, "step_frac": step_gbs / peak,
                "algo_bytes_per_cell_step": step_bpc,
                # S:8(d): fractions also against the north_star's ~8 TB/s nominal
                "nominal_peak": NOMINAL_HBM_GBS, "frac_nominal": ach / NOMINAL_HBM_GBS if ach else None,
                "step_frac_nominal": step_gbs / NOMINAL_HBM_GBS}
    win = ncu_window(nx // px, ny // py)
    if win:
        win["frac"] = win["hbm_gbs"] / peak
        win["frac_nominal"] = win["hbm_gbs"] / NOMINAL_HBM_GBS
        roofline["ncu_window"] = win
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    roofline["alu"] = issue_roofline(kernels, top, clk.get("sm_mhz"), nsm)

    # end-to-end through the host-buffer C-ABI entry (pinned host memory)
    e2e = None
    if not args.no_e2e and world == 1:
        nc, nn = cells, (nx + 1) * (ny + 1)
        host = {}
        for name, shp in (("density0", (ny, nx)), ("energy0", (ny, nx)),
                          ("xvel0", (ny + 1, nx + 1)), ("yvel0", (ny + 1, nx + 1))):
            host[name] = torch.empty(shp, dtype=torch.float64, pin_memory=True).numpy()
        for name in host:  # current state as the input
            host[name][...] = sim.read(name)
        ke = max(3, min(args.steps, 10))
        sim.step_host(1, host, host)  # warm
        t0 = time.perf_counter()
        for _ in range(ke):
            sim.step_host(1, host, host)
        te = time.perf_counter() - t0
        e2e = {"value": cells * ke / te, "unit": UNIT, "h2d_bytes_per_step": 8 * (2 * nc + 2 * nn),
               "d2h_bytes_per_step": 8 * (2 * nc + 2 * nn), "steps": ke,
               "api": "clover_step_host (h2d state, 1 step, d2h state)"}
        # the same entry point as a user runs a simulation: state in once, K
        # steps, state out once (per-step bytes amortised over the K steps)
        t0 = time.perf_counter()
        sim.step_host(args.steps, host, host)
        tk = time.perf_counter() - t0
        e2e["run"] = {"value": cells * args.steps / tk, "unit": UNIT, "steps": args.steps,
                      "h2d_bytes_per_step": 8 * (2 * nc + 2 * nn) / args.steps,
                      "d2h_bytes_per_step": 8 * (2 * nc + 2 * nn) / args.steps,
                      "api": f"clover_step_host (h2d state, {args.steps} steps, d2h state)"}

    if not args.no_e2e and world > 1:
        # every rank moves its own strip of the global host arrays through
        # clover_step_host (collective): the arrays are allocated lazily
        # (np.empty), only this rank's rows are touched and pinned
        # (cudaHostRegister); wall clock per call, max over ranks
        gj0, gk0, bw, bh = sim.local_block()
        host, regs = {}, []
        for name, shp in (("density0", (ny, nx)), ("energy0", (ny, nx)),
                          ("xvel0", (ny + 1, nx + 1)), ("yvel0", (ny + 1, nx + 1))):
            a = np.empty(shp, dtype=np.float64)
            host[name] = a
            r1 = min(shp[0], gk0 + bh + 1)
            ptr = a.ctypes.data + gk0 * a.strides[0]
            nbytes = (r1 - gk0) * a.strides[0]
            if torch.cuda.cudart().cudaHostRegister(ptr, nbytes, 0) == 0:
                regs.append(ptr)
        sim.step_host(0, {}, host)  # this rank's rows <- the current state
        ke = max(3, min(args.steps, 10))
        sim.step_host(1, host, host)  # warm
        dist.barrier()
        t0 = time.perf_counter()
        for _ in range(ke):
            sim.step_host(1, host, host)
        te = cdist.max_over_ranks(time.perf_counter() - t0, None if host_tp else dev)
        for ptr in regs:
            torch.cuda.cudart().cudaHostUnregister(ptr)
        nc, nn = cells, (nx + 1) * (ny + 1)
        e2e = {"value": cells * ke / te, "unit": UNIT, "h2d_bytes_per_step": 8 * (2 * nc + 2 * nn),
               "d2h_bytes_per_step": 8 * (2 * nc + 2 * nn), "steps": ke,
               "api": "clover_step_host (each rank: h2d its strip of the state, 1 step, d2h), "
                      "bytes summed over ranks",
               "pinned": len(regs) == 4}

    # side measurement: the same mesh with every cell moving (seeded smooth
    # random state + noise, workloads.random_state_fields), so the headline
    # is not an artifact of the bm deck's quiescent regions
    active = None
    if world == 1 and not args.no_active:
        from workloads import random_state_fields
        adeck = bm_deck(nx, ny)
        adeck["max_timestep"] = 1.0
        sim.close()
        act = Clover(adeck, stream=stream)
        act.load_state(random_state_fields(7, nx, ny, smooth=True))
        act.step(args.warmup)
        act.sync()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a0.record(stream)
        act.step(args.steps)
        a1.record(stream)
        torch.cuda.synchronize()
        act.sync()
        ams = a0.elapsed_time(a1) / args.steps
        active = {"ms_per_step": ams, "value": cells / (ams / 1e3), "unit": UNIT,
                  "state": "workloads.random_state_fields(7, smooth=True): every cell moving, limiters active"}
        act.close()
        sim = Clover(deck, px=px, py=py, rank=rank, nranks=world, unique_id=uid, stream=stream,
                     host_transport=ht)
        sim.step(args.steps + args.warmup)

    # full configs[2] run: all 300 steps from step 0, each on a
    # freshly initialised context (median of 3, after one warm-up context);
    # covers the late, fully developed flow as well as the cheap early steps
    full = None
    if world == 1 and not args.no_full and not args.mesh and not args.strong:
        sim.close()
        nfull = 300
        times = []
        for rep in range(4):
            f = Clover(deck, stream=stream)
            f.sync()
            f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            f0.record(stream)
            f.step(nfull)
            f1.record(stream)
            torch.cuda.synchronize()
            f.sync()
            if rep:
                times.append(f0.elapsed_time(f1))
            f.close()
        fms = statistics.median(times)
        full = {"steps": nfull, "ms": fms, "ms_per_step": fms / nfull,
                "value": cells * nfull / (fms / 1e3), "unit": UNIT, "repeats_ms": times,
                "how": "clover_step(ctx, 300) from step 0 on a fresh context, CUDA events, "
                       "median of 3 after one warm-up context (graphs on)"}
        sim = Clover(deck, px=px, py=py, rank=rank, nranks=world, unique_id=uid, stream=stream,
                     host_transport=ht)
        sim.step(args.steps + args.warmup)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cdeck = bm_deck(nx, ny)
        rate, t = oracle_rate(cdeck, 6)
        cpu = {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"first 6 steps of the same {nx}x{ny} bm workload, single-threaded "
                         f"C++ oracle (-O2), {t:.1f} s"}
        cpu.update(host_cpu())

    summ = sim.field_summary()
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
                "higher_is_better": True, "scaling": "strong" if args.strong else "weak",
                "vs_baseline": None,
                "dtype": "f64", "data": "synthetic",
                "config": {"workload": ("configs[3]: CloverLeaf 2D bm deck 7680x7680 strong-scaled"
                                        if args.strong else
                                        "configs[2]: CloverLeaf 2D bm deck 3840x3840 (clover_bm16 shape), "
                                        "1 GPU bandwidth-roofline run" if world == 1 else
                                        f"configs[4]: weak scaling, 3840^2 cells per GPU, global {nx}x{ny} "
                                        f"on [0,10]^2 (reading A4)"),
                           "mesh": [nx, ny], "decomposition": f"{px}x{py}",
                           "transport": (("nccl, device-initiated LSA halo stores"
                                          if os.environ.get("CLOVER_LSA", "0") != "0" else "nccl")
                                         if not host_tp else "host (gloo; not a bench value)")
                           if world > 1 else None,
                           "halo_exchange": ("deep: 1 state exchange (7 rows) + dt MIN per step"
                                             if deep_halo else "per phase") if world > 1 else None,
                           "l2": "inputs larger than L2 (18 fp64 fields of the mesh, >2 GB vs 126 MB L2)",
                           "graphs": not host_tp},
                "gpu_launches": launches,
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "clocks": clk,
                "kernels": kernels,
                "active_flow": active,
                "full_run": full,
                "paper_context": PAPER_CONTEXT,
                "summary_after": summ}
        print(json.dumps(line), flush=True)
    sim.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
