"""Aggregate an ncu `--page source --print-source sass --csv` dump by opcode:
python scripts/sass_mix.py dump.csv  -> executed warp instructions per opcode
and the stall samples attributed to each opcode."""
import csv
import collections
import sys

rows = list(csv.reader(open(sys.argv[1])))
i0 = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[i0]
ie, ss = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
cnt, stall = collections.Counter(), collections.Counter()
for r in rows[i0 + 1:]:
    if len(r) <= ie or not r[ie].replace(",", "").isdigit():
        continue
    src = r[h.index("Source")].strip()
    op = src.split()[0] if src else "?"
    if op.startswith("@"):
        op = src.split()[1]
    op = op.split(".")[0]
    cnt[op] += int(r[ie].replace(",", ""))
    stall[op] += int(r[ss].replace(",", "") or 0)
tot, st = sum(cnt.values()), sum(stall.values())
print(f"total warp inst {tot:,}  stall samples {st:,}")
for op, n in cnt.most_common(30):
    print(f"{op:10s} {n:14,d} {100 * n / tot:5.1f}%  stall {100 * stall[op] / max(st, 1):5.1f}%")
