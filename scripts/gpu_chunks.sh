mkdir -p gpurun_out
rm -f gpurun_out/chunks.jsonl
for a in "7680 7680 1 8" "7680 7680 2 4" "7680 7680 1 4" "7680 7680 2 2" "7680 7680 1 2" "3840 7680 1 2"; do
  timeout 300 python scripts/chunk_overhead.py $a 20 >> gpurun_out/chunks.jsonl 2>> gpurun_out/chunks.err
done
cat gpurun_out/chunks.jsonl; tail -3 gpurun_out/chunks.err
