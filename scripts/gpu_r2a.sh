# Round-2 GPU pass A: GPU test suite, bench line, fp64 peaks, sanitizers.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2a_smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r2a_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2a_pytest.log
tail -3 gpurun_out/r2a_pytest.log
timeout 600 python bench.py > gpurun_out/r2a_bench.json 2> gpurun_out/r2a_bench.err
tail -c 1500 gpurun_out/r2a_bench.json
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/fp64_peak scripts/fp64_peak.cu && /tmp/fp64_peak > gpurun_out/r2a_fp64_peaks.jsonl
cat gpurun_out/r2a_fp64_peaks.jsonl
for tool in memcheck racecheck synccheck; do
  for c in bm chunks; do
    timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_run.py $c > gpurun_out/r2a_san_${tool}_${c}.log 2>&1
    echo "$tool $c rc=$?"; tail -3 gpurun_out/r2a_san_${tool}_${c}.log
  done
done
