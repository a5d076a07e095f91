# library variants (build_ab/) on several meshes: kernel_times graph step
# time, bm deck, two interleaved repeats.  VARIANTS="a b" MESHES="NX:NY ..."
mkdir -p gpurun_out
: > gpurun_out/mesh_ab.jsonl
for r in 1 2; do
  for m in ${MESHES:-7680:960 3840:3840}; do
    nx=${m%:*}; ny=${m#*:}
    for v in ${VARIANTS:-base}; do
      echo -n "{\"variant\": \"$v\", \"r\": $r, \"t\": " >> gpurun_out/mesh_ab.jsonl
      CLOVER_LIB=build_ab/libclover_$v.so timeout 300 python scripts/kernel_times.py $nx $ny 40 | tr -d '\n' >> gpurun_out/mesh_ab.jsonl 2>&1
      echo "}" >> gpurun_out/mesh_ab.jsonl
    done
  done
done
python - <<'PY'
import json
for l in open("gpurun_out/mesh_ab.jsonl"):
    try: d = json.loads(l)
    except Exception: print("BAD", l[:200]); continue
    t = d["t"]; k = t["kernels_ms"]
    print(f'{d["variant"]:6s} {t["mesh"]} {t["ms_per_step_graphs"]:.4f}', " ".join(f'{n.replace("k_advec_","").replace("k_","")}={v:.4f}' for n, v in k.items() if v > 0.005))
PY
