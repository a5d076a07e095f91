# single-chunk A/B against the pre-change library, then the whole GPU suite
mkdir -p gpurun_out
: > gpurun_out/deep_ab.jsonl
for r in 1 2 3; do
  for v in base new; do
    lib=build_ab/libclover_base.so; [ $v = new ] && lib=paper_conf_cluster_regulymg15_b200/libclover.so
    echo -n "{\"variant\": \"$v\", \"r\": $r, \"t\": " >> gpurun_out/deep_ab.jsonl
    CLOVER_LIB=$lib timeout 300 python scripts/kernel_times.py 3840 3840 40 | tr -d '\n' >> gpurun_out/deep_ab.jsonl 2>&1
    echo "}" >> gpurun_out/deep_ab.jsonl
  done
done
python - <<'PY'
import json
for l in open("gpurun_out/deep_ab.jsonl"):
    try: d = json.loads(l)
    except Exception: print("BAD", l[:300]); continue
    t = d["t"]; k = t["kernels_ms"]
    print(f'{d["variant"]:5s} {t["ms_per_step_graphs"]:.4f}', " ".join(f'{n.replace("k_advec_","").replace("k_","")}={v:.4f}' for n, v in k.items() if v > 0.01))
PY
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest.log
tail -3 gpurun_out/pytest.log
grep -E "^FAILED|^ERROR" gpurun_out/pytest.log | head -20
