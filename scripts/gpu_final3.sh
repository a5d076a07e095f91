# end of round 2: profiles (bench, launch list, ncu full capture, NCCL launch list),
# GPU suite, smoke, configs lines (960^2, 7680^2 strong base) and the 1x8 / 1x2
# multi-chunk proxies of the strong-scaling ranks
bash scripts/profile_round.sh
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest.log
tail -3 gpurun_out/pytest.log
grep -E "^FAILED|^ERROR" gpurun_out/pytest.log | head -20
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -2 gpurun_out/smoke.log
bash scripts/configs_run.sh
: > gpurun_out/chunks_final.jsonl
for cfg in "7680 7680 1 8" "3840 7680 1 2"; do
  timeout 600 python scripts/chunk_overhead.py $cfg 2>/dev/null | grep '^{' >> gpurun_out/chunks_final.jsonl
done
python - <<'PY'
import json
for l in open("gpurun_out/chunks_final.jsonl"):
    d = json.loads(l)
    print(d["mesh"], d["chunks"], "one", round(d["one_chunk_ms"], 3), "rank alone", round(d["rank_chunk_alone_ms"], 3),
          "bound", round(d["strong_scaling_efficiency_bound"], 3))
PY
