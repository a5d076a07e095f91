# device-initiated halo stores (NCCL symmetric window + LSA barrier): tests,
# then the chunk-overhead comparison
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -p no:cacheprovider -k "lsa" -x > gpurun_out/pytest_lsa.log 2>&1
echo "pytest lsa rc=$?" >> gpurun_out/pytest_lsa.log
tail -30 gpurun_out/pytest_lsa.log
: > gpurun_out/lsa_chunks.jsonl
for cfg in "7680 7680 1 8" "7680 7680 1 4" "7680 7680 1 2"; do
  timeout 600 python scripts/chunk_overhead.py $cfg >> gpurun_out/lsa_chunks.jsonl 2>&1
done
python - <<'PY'
import json
for l in open("gpurun_out/lsa_chunks.jsonl"):
    try: d = json.loads(l)
    except Exception: print(l[:300]); continue
    print(d["mesh"], d["chunks"], "one %.3f" % d["one_chunk_ms"], " ".join(f'{k}={d[k]["ms"]:.3f}' for k in d if isinstance(d[k], dict)))
PY
