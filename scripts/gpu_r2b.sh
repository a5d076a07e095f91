# Round-2 GPU pass B: GPU tests, chunk-overhead (virtual multi-GPU) table.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2b_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2b_pytest.log
tail -3 gpurun_out/r2b_pytest.log
grep -E "^FAILED|^ERROR" gpurun_out/r2b_pytest.log | head -20
for a in "7680 7680 1 8" "3840 7680 1 2" "7680 7680 2 4" "7680 7680 1 2" "7680 7680 1 4"; do
  timeout 300 python scripts/chunk_overhead.py $a 20 >> gpurun_out/r2b_chunks.jsonl 2>> gpurun_out/r2b_chunks.err
done
cat gpurun_out/r2b_chunks.jsonl; tail -5 gpurun_out/r2b_chunks.err
