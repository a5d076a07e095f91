# Per-kernel durations (ncu, serialised) of A/B library variants:
# bash scripts/ab_ncu.sh NAME...   (libraries from build_ab/libclover_NAME.so)
mkdir -p gpurun_out
for n in "$@"; do
  CLOVER_LIB=build_ab/libclover_$n.so timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none \
    -s 200 -c 200 --csv --log-file gpurun_out/abn_$n.csv python scripts/prof_run.py 3840 3840 30 > /dev/null 2>&1
  python - "$n" <<'PY'
import csv, io, sys, collections
n = sys.argv[1]
lines = [l for l in open(f"gpurun_out/abn_{n}.csv") if l.startswith('"')]
rows = list(csv.reader(io.StringIO("".join(lines))))
h = rows[0]
k, v = h.index("Kernel Name"), h.index("Metric Value")
t = collections.defaultdict(list)
for r in rows[1:]:
    t[r[k].split("(")[0].replace("void ", "").replace("clover::", "")].append(float(r[v].replace(",", "")))
print(n, "  ".join(f"{a}={sum(b)/len(b)/1e3:.1f}us" for a, b in sorted(t.items())))
PY
done
