mkdir -p gpurun_out
timeout 120 python __graft_entry__.py smoke > gpurun_out/flow_smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/flow_smoke.log
rm -f gpurun_out/quick.jsonl
for i in 1 2; do timeout 120 python scripts/kernel_times.py 3840 3840 40 >> gpurun_out/quick.jsonl 2>>gpurun_out/quick.err; echo "kt rc=$?"; done
cat gpurun_out/quick.jsonl | cut -c1-400
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest.log; grep -E "^FAILED|^E  " gpurun_out/pytest.log | head -5
