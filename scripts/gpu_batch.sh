# batched chunk launches: multi-chunk tests, then chunk overhead with and
# without batching (CLOVER_BATCH=0)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "chunk or deep or lsa or nccl or remote or overlap or decomposition or batched" > gpurun_out/pytest_batch.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_batch.log
tail -3 gpurun_out/pytest_batch.log; grep -E "^FAILED|^ERROR|Error" gpurun_out/pytest_batch.log | head
: > gpurun_out/batch_chunks.jsonl
for b in 1 0; do
  for cfg in "7680 7680 1 8" "3840 7680 1 2"; do
    echo -n "{\"batch\": $b, \"r\": " >> gpurun_out/batch_chunks.jsonl
    CLOVER_BATCH=$b timeout 600 python scripts/chunk_overhead.py $cfg | tr -d '\n' >> gpurun_out/batch_chunks.jsonl 2>&1
    echo "}" >> gpurun_out/batch_chunks.jsonl
  done
done
python - <<'PY'
import json
for l in open("gpurun_out/batch_chunks.jsonl"):
    try: d = json.loads(l)
    except Exception: print(l[:300]); continue
    r = d["r"]
    print("batch", d["batch"], r["mesh"], r["chunks"], "one %.3f" % r["one_chunk_ms"], " ".join(f'{k}={r[k]["ms"]:.3f}' for k in r if isinstance(r[k], dict)))
PY
