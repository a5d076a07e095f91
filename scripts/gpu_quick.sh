# quick A/B: per-kernel times (3840^2 bm, 2 repeats) then the GPU test suite
mkdir -p gpurun_out; rm -f gpurun_out/quick.jsonl
for i in 1 2; do timeout 300 python scripts/kernel_times.py 3840 3840 40 >> gpurun_out/quick.jsonl 2>>gpurun_out/quick.err; done
cat gpurun_out/quick.jsonl
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider ${PYTEST_ARGS} > gpurun_out/pytest.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/pytest.log; grep -E "^FAILED|^E  " gpurun_out/pytest.log | head -5
