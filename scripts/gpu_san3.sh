# compute-sanitizer on the batched multi-chunk launches (2x2 chunks and 1x3
# deep-halo strips are batched by default)
mkdir -p gpurun_out
: > gpurun_out/san3.txt
for tool in memcheck racecheck synccheck; do
  for c in chunks deep; do
    echo "== $tool $c (batched)" >> gpurun_out/san3.txt
    timeout 900 compute-sanitizer --tool $tool python scripts/sanitize_run.py $c > gpurun_out/san3_${tool}_$c.log 2>&1
    echo "rc=$?" >> gpurun_out/san3.txt
    grep -E "sanitize_run|SUMMARY" gpurun_out/san3_${tool}_$c.log >> gpurun_out/san3.txt
  done
done
cat gpurun_out/san3.txt
