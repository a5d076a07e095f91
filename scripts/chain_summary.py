"""Summarise gpurun_out/chain_ab.jsonl (kernel_times per variant) and the
ncu DRAM reads of gpurun_out/chain_ncu_{base,chain0}.csv."""
import csv
import json
import re
import sys

txt = open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/chain_ab.jsonl").read()
for m in re.finditer(r'\{"variant": "(\w+)", "mode": "(\w+)", "r": (\d), "t": (\{.*?\})\s*\n\}', txt, re.S):
    t = json.loads(m.group(4))
    k = t["kernels_ms"]
    print(f'{m.group(1):8s} {m.group(2):6s} {t["ms_per_step_graphs"]:.4f}',
          " ".join(f'{n.replace("k_advec_", "").replace("k_", "")}={v:.4f}' for n, v in k.items() if v > 0.01))
alg = {"ks_visc_dt": 32, "ks_lagrangian": 40, "ks_advec_x<1>": 48, "ks_advec_x<2>": 40,
       "ks_advec_y<1>": 48, "ks_advec_y<2>": 40}
res = {}
for v in ("chain0", "base"):
    rows = list(csv.reader(l for l in open(f"gpurun_out/chain_ncu_{v}.csv") if l.startswith('"')))
    h = rows[0]
    ik, im, iv, iid = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
    d = {}
    for r in rows[1:]:
        d.setdefault((r[iid], r[ik].replace("void ", "").split("(")[0]), {})[r[im]] = float(r[iv].replace(",", ""))
    for (i, k), mm in d.items():
        res.setdefault(k, {}).setdefault(v, []).append((mm["dram__bytes_read.sum"] / 1e6, mm["gpu__time_duration.sum"] / 1e3))
cells = 3840 * 3840
print("| kernel | row layout MB / us | band layout MB / us | algorithmic MB | read ratio |")
print("|---|---|---|---|---|")
for k, vv in res.items():
    a = [sum(x) / len(x) for x in zip(*vv["chain0"])]
    b = [sum(x) / len(x) for x in zip(*vv["base"])]
    al = alg[k] * cells / 1e6
    print(f"| {k} | {a[0]:.0f} / {a[1]:.1f} | {b[0]:.0f} / {b[1]:.1f} | {al:.0f} | {a[0]/al:.3f} -> {b[0]/al:.3f} |")
