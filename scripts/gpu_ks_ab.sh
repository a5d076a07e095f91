# rows-per-segment A/B: kernel_times (bm 3840^2 and seeded active flow) per
# library variant in build_ab/, two interleaved repeats
mkdir -p gpurun_out
: > gpurun_out/ks_ab.jsonl
for r in 1 2; do
  for v in ${VARIANTS:-base yks64 xks32 lks32 vks64}; do
    for mode in bm active; do
      a=""; [ $mode = active ] && a=active
      echo -n "{\"variant\": \"$v\", \"mode\": \"$mode\", \"r\": $r, \"t\": " >> gpurun_out/ks_ab.jsonl
      CLOVER_LIB=build_ab/libclover_$v.so timeout 300 python scripts/kernel_times.py 3840 3840 40 $a >> gpurun_out/ks_ab.jsonl 2>&1
      echo "}" >> gpurun_out/ks_ab.jsonl
    done
  done
done
python - <<'PY'
import json
for l in open("gpurun_out/ks_ab.jsonl"):
    try: d = json.loads(l)
    except Exception: print("BAD", l[:200]); continue
    t = d["t"]; k = t["kernels_ms"]
    print(f'{d["variant"]:8s} {d["mode"]:6s} {t["ms_per_step_graphs"]:.4f}', " ".join(f'{n.replace("k_advec_","").replace("k_","")}={v:.4f}' for n, v in k.items() if v > 0.01))
PY
