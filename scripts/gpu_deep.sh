# deep halos: new GPU tests first, then single-chunk A/B against the
# pre-change library (build_ab/libclover_base.so), chunk overhead with deep
# variants, then the whole GPU suite
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "deep or kernels_per_step" > gpurun_out/pytest_deep.log 2>&1
echo "pytest deep rc=$?" >> gpurun_out/pytest_deep.log
tail -3 gpurun_out/pytest_deep.log
grep -E "^FAILED|^ERROR|Error" gpurun_out/pytest_deep.log | head -20
: > gpurun_out/deep_ab.jsonl
for r in 1 2; do
  for v in base new; do
    lib=build_ab/libclover_base.so; [ $v = new ] && lib=paper_conf_cluster_regulymg15_b200/libclover.so
    echo -n "{\"variant\": \"$v\", \"r\": $r, \"t\": " >> gpurun_out/deep_ab.jsonl
    CLOVER_LIB=$lib timeout 300 python scripts/kernel_times.py 3840 3840 40 | tr -d '\n' >> gpurun_out/deep_ab.jsonl 2>&1
    echo "}" >> gpurun_out/deep_ab.jsonl
  done
done
cat gpurun_out/deep_ab.jsonl | cut -c1-200
: > gpurun_out/deep_chunks.jsonl
for cfg in "7680 7680 1 8" "7680 7680 1 4" "7680 7680 1 2" "3840 7680 1 2"; do
  timeout 600 python scripts/chunk_overhead.py $cfg >> gpurun_out/deep_chunks.jsonl 2>&1
done
python - <<'PY'
import json
for l in open("gpurun_out/deep_chunks.jsonl"):
    try: d = json.loads(l)
    except Exception: print(l[:300]); continue
    print(d["mesh"], d["chunks"], "one %.3f" % d["one_chunk_ms"], " ".join(f'{k}={d[k]["ms"]:.3f}' for k in d if isinstance(d[k], dict)))
PY
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest.log
tail -3 gpurun_out/pytest.log
grep -E "^FAILED|^ERROR" gpurun_out/pytest.log | head -20
