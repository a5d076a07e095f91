# f2 fold A/B: per-kernel and graph step times at 3840^2 (bm, 40 steps after
# 20) with CLOVER_FOLD=0/1, twice; then the GPU suite with the fold on
mkdir -p gpurun_out
: > gpurun_out/fold_ab.jsonl
for r in 1 2; do
  for f in 0 1; do
    echo -n "{\"fold\": $f, \"r\": $r, \"t\": " >> gpurun_out/fold_ab.jsonl
    CLOVER_FOLD=$f timeout 300 python scripts/kernel_times.py 3840 3840 40 >> gpurun_out/fold_ab.jsonl 2>&1
    echo "}" >> gpurun_out/fold_ab.jsonl
  done
done
cat gpurun_out/fold_ab.jsonl
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider ${PYTEST_ARGS} > gpurun_out/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest.log
tail -3 gpurun_out/pytest.log
grep -E "^FAILED|^ERROR" gpurun_out/pytest.log | head -30
