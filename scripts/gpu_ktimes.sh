mkdir -p gpurun_out; rm -f gpurun_out/ktimes.jsonl
for a in "7680 7680" "7680 3840" "7680 1920" "7680 960" "3840 3840" "1920 1920" "960 960"; do
  timeout 300 python scripts/kernel_times.py $a 30 active >> gpurun_out/ktimes.jsonl 2>> gpurun_out/ktimes.err
done
cat gpurun_out/ktimes.jsonl
