# compute-sanitizer on the deep-halo views and the LSA transport, then the GPU suite
mkdir -p gpurun_out
: > gpurun_out/san2.txt
for tool in memcheck racecheck synccheck; do
  for c in deep lsa; do
    [ $c = lsa ] && [ $tool != memcheck ] && continue
    echo "== $tool $c" >> gpurun_out/san2.txt
    timeout 900 compute-sanitizer --tool $tool python scripts/sanitize_run.py $c > gpurun_out/san_${tool}_$c.log 2>&1
    echo "rc=$?" >> gpurun_out/san2.txt
    grep -E "sanitize_run|SUMMARY" gpurun_out/san_${tool}_$c.log >> gpurun_out/san2.txt
  done
done
cat gpurun_out/san2.txt
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest.log
tail -3 gpurun_out/pytest.log
grep -E "^FAILED|^ERROR" gpurun_out/pytest.log | head -20
