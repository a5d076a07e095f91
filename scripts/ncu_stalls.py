"""Per-kernel summary of an ncu --set full report: time, DRAM GB/s, issue
and fp64-pipe utilisation, occupancy and the main stall reasons (cycles per
issued instruction).  usage: python scripts/ncu_stalls.py REPORT.ncu-rep"""
import csv
import io
import subprocess
import sys

raw = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "raw", "--csv"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, u, data = rows[0], rows[1], rows[2:]


def g(r, c):
    try:
        return float(r[h.index(c)].replace(",", ""))
    except (ValueError, IndexError):
        return float("nan")


stalls = ["long_scoreboard", "wait", "not_selected", "math_pipe_throttle", "short_scoreboard",
          "dispatch_stall", "branch_resolving", "no_instruction", "barrier", "lg_throttle", "mio_throttle"]
print(f"{'kernel':22s} {'us':>6s} {'GB/s':>6s} {'iss%':>5s} {'fp64%':>5s} {'warps':>5s} {'regs':>4s} " +
      " ".join(f"{s[:6]:>6s}" for s in stalls))
for r in data:
    n = r[h.index("Kernel Name")].split("(")[0].replace("void ", "").replace("clover::", "")
    t = g(r, "gpu__time_duration.sum")
    tu = u[h.index("gpu__time_duration.sum")]
    tns = t * {"ns": 1, "nsecond": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6}.get(tu, 1)
    sc = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u[h.index("dram__bytes_read.sum")], 1)
    gbs = (g(r, "dram__bytes_read.sum") + g(r, "dram__bytes_write.sum")) * sc / tns
    st = [g(r, f"smsp__average_warps_issue_stalled_{s}_per_issue_active.ratio") for s in stalls]
    print(f"{n[:22]:22s} {tns / 1e3:6.1f} {gbs:6.0f} {g(r, 'smsp__issue_active.avg.pct_of_peak_sustained_active'):5.1f} "
          f"{g(r, 'sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active'):5.1f} "
          f"{g(r, 'sm__warps_active.avg.pct_of_peak_sustained_active'):5.1f} {g(r, 'launch__registers_per_thread'):4.0f} " +
          " ".join(f"{x:6.2f}" for x in st))
