"""Per-CUDA-source-line instruction counts and stall samples from an ncu
`--page source --print-source cuda,sass --csv` dump (several files):
python scripts/src_lines.py dump.csv [N] -> the N hottest source lines."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
fname = ""
hdr = None
acc = {}
tot_i = tot_s = 0
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or r[0] == "Function Name":
        continue
    if r[0] != "":  # a source line row (aggregated)
        try:
            ie = int(r[hdr.index("Instructions Executed")].replace(",", "") or 0)
            st = int(r[hdr.index("Warp Stall Sampling (All Samples)")].replace(",", "") or 0)
        except ValueError:
            continue
        key = (fname, int(r[0]))
        a = acc.setdefault(key, [0, 0, r[1][:90]])
        a[0] += ie
        a[1] += st
        tot_i += ie
        tot_s += st
print(f"total warp inst {tot_i:,}  stall samples {tot_s:,}")
for (f, ln), (i, s, src) in sorted(acc.items(), key=lambda kv: -kv[1][0])[:n]:
    print(f"{100 * i / tot_i:5.1f}% {100 * s / max(tot_s, 1):5.1f}%st {f}:{ln:<5d} {src}")
