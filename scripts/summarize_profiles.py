"""Turn the ncu outputs of scripts/profile_round.sh into committed summaries:
profiles/<tag>_launches.csv (per-launch kernel list of the bench command),
profiles/<tag>_kernels.md (per-kernel table from the --set full capture) and
profiles/ncu_traffic.json (DRAM bytes per launch, read by bench.py)."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1] if len(sys.argv) > 1 else "r1"
G = os.path.join(ROOT, "gpurun_out")
P = os.path.join(ROOT, "profiles")
os.makedirs(P, exist_ok=True)
NAMES = {"ks_visc_dt": "k_visc_dt", "ks_lagrangian": "k_lagrangian"}


def short(name):
    n = name.split("(")[0].replace("void ", "").replace("clover::", "")
    for a, b in (("ks_advec_cell_x<1>", "k_advec_cell_x<1>"), ("ks_advec_cell_x<2>", "k_advec_cell_x<2>"),
                 ("ks_advec_cell_y<1>", "k_advec_cell_y<1>"), ("ks_advec_cell_y<2>", "k_advec_cell_y<2>"),
                 ("ks_advec_mom_x<1>", "k_advec_mom_x<1>"), ("ks_advec_mom_x<2>", "k_advec_mom_x<2>"),
                 ("ks_advec_mom_y<1>", "k_advec_mom_y<1>"), ("ks_advec_mom_y<2>", "k_advec_mom_y<2>"),
                 ("ks_advec_x<1>", "k_advec_x<1>"), ("ks_advec_x<2>", "k_advec_x<2>"),
                 ("ks_advec_y<1>", "k_advec_y<1>"), ("ks_advec_y<2>", "k_advec_y<2>"),
                 ("ks_cell_y_walls<1>", "k_cell_y_walls<1>"), ("ks_cell_y_walls<2>", "k_cell_y_walls<2>")):
        if n.startswith(a):
            return b
    return NAMES.get(n, n)


# launch list
src = os.path.join(G, "launches.csv")
if os.path.exists(src):
    lines = [l for l in open(src) if l.startswith('"')]
    rows = list(csv.reader(io.StringIO("".join(lines))))
    hdr, data = rows[0], rows[1:]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    per = {}
    order = []
    for r in data:
        key = (r[0], short(r[ki]))
        if key not in per:
            per[key] = {}
            order.append(key)
        per[key][r[mi]] = float(r[vi].replace(",", ""))
    with open(os.path.join(P, f"{tag}_launches.csv"), "w") as fh:
        fh.write("launch,kernel,gpu_time_ns,dram_read_bytes,dram_write_bytes\n")
        for key in order:
            m = per[key]
            fh.write(f"{key[0]},{key[1]},{m.get('gpu__time_duration.sum', 0):.0f},"
                     f"{m.get('dram__bytes_read.sum', 0):.0f},{m.get('dram__bytes_write.sum', 0):.0f}\n")
    print("wrote launches", len(order))

# NCCL virtual-remote launch list (kernel name, duration): NCCL's own kernels
src = os.path.join(G, "launches_nccl.csv")
if os.path.exists(src):
    lines = [l for l in open(src) if l.startswith('"')]
    rows = list(csv.reader(io.StringIO("".join(lines))))
    hdr, data = rows[0], rows[1:]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    with open(os.path.join(P, f"{tag}_launches_nccl.csv"), "w") as fh:
        fh.write("launch,kernel,gpu_time_ns\n")
        for r in data:
            if r[mi] == "gpu__time_duration.sum":
                fh.write(f"{r[0]},{r[ki].split('(')[0]},{r[vi].replace(',', '')}\n")
    print("wrote nccl launches")

# full capture
rep = os.path.join(G, "prof_full.ncu-rep")
if os.path.exists(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, data = rows[0], rows[1], rows[2:]

    def g(r, c):
        try:
            v = r[hdr.index(c)].replace(",", "")
            return float(v)
        except (ValueError, IndexError):
            return None
    cells = 3840 * 3840
    kern = {}
    md = [f"# ncu --set full summary ({tag}): bm 3840x3840, one launch per kernel type\n",
          "Captured with `ncu --set full --clock-control none --import-source on -k regex:ks_` on "
          "`scripts/prof_run.py 3840 3840 54` with `-s 200 -c 12`: steps 51-53, x-first, y-first, x-first (scripts/profile_round.sh). DRAM bytes in MB "
          "(units as reported: " + units[hdr.index('dram__bytes_read.sum')] + ").\n",
          "| kernel | time us | DRAM read | DRAM write | DRAM GB/s | issue % | fp64 pipe % | warps active % | regs | thread inst/cell |",
          "|---|---|---|---|---|---|---|---|---|---|"]
    tunit = units[hdr.index("gpu__time_duration.sum")]
    tscale = {"ns": 1.0, "nsecond": 1.0, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6}.get(tunit, 1.0)
    for r in data:
        n = short(r[hdr.index("Kernel Name")])
        t = g(r, "gpu__time_duration.sum") * tscale  # ns
        rd, wr = g(r, "dram__bytes_read.sum"), g(r, "dram__bytes_write.sum")
        unit = units[hdr.index("dram__bytes_read.sum")]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
        inst = g(r, "smsp__inst_executed.sum")
        md.append(f"| {n} | {t / 1e3 if t else 0:.1f} | {rd:.1f} | {wr:.1f} | {(rd + wr) * scale / (t * 1e-9) / 1e9:.0f} | "
                  f"{g(r, 'smsp__issue_active.avg.pct_of_peak_sustained_active'):.1f} | "
                  f"{g(r, 'sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active'):.1f} | "
                  f"{g(r, 'sm__warps_active.avg.pct_of_peak_sustained_active'):.1f} | "
                  f"{g(r, 'launch__registers_per_thread'):.0f} | {inst * 32 / cells:.0f} |")
        kern.setdefault(n, []).append({"dram_bytes": (rd + wr) * scale, "time_ns": t, "inst": inst,
                                       "issue": g(r, 'smsp__issue_active.avg.pct_of_peak_sustained_active'),
                                       "fp64": g(r, 'sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active')})
    with open(os.path.join(P, f"{tag}_kernels.md"), "w") as fh:
        fh.write("\n".join(md) + "\n")
    allx = [x for v in kern.values() for x in v]
    tb, tt = sum(x["dram_bytes"] for x in allx), sum(x["time_ns"] for x in allx)
    out = {"mesh": [3840, 3840], "source": f"profiles/{tag}_kernels.md (ncu --set full)",
           "kernels": {k: {"dram_bytes_per_launch": sum(x["dram_bytes"] for x in v) / len(v),
                           "launches": len(v)} for k, v in kern.items()},
           # S:8(d) hbm_gbs: sum of DRAM bytes over sum of kernel time, the
           # streaming kernels of the captured window (cold-cache, serialised)
           "window": {"launches": len(allx), "dram_bytes": tb, "time_ns": tt,
                      "hbm_gbs": tb / (tt * 1e-9) / 1e9 if tt else None}}
    with open(os.path.join(P, "ncu_traffic.json"), "w") as fh:
        json.dump(out, fh, indent=1)
    avg = lambda v, k: sum(x[k] for x in v) / len(v)
    ins = {"mesh": [3840, 3840], "source": f"profiles/{tag}_kernels.md (ncu --set full, smsp__inst_executed.sum)",
           "kernels": {k: {"warp_inst_per_launch": avg(v, "inst"),
                           "thread_inst_per_cell": avg(v, "inst") * 32 / cells,
                           "issue_active_pct": avg(v, "issue"), "fp64_pipe_pct": avg(v, "fp64"),
                           "launches": len(v)} for k, v in kern.items()}}
    with open(os.path.join(P, "ncu_instr.json"), "w") as fh:
        json.dump(ins, fh, indent=1)
    print("wrote kernels", len(kern))
b = os.path.join(G, "bench.json")
if os.path.exists(b):
    line = open(b).read().strip().splitlines()[-1]
    with open(os.path.join(P, f"{tag}_bench.json"), "w") as fh:
        fh.write(line + "\n")
    print("wrote bench")
