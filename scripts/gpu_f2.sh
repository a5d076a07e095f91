mkdir -p gpurun_out
for i in 1 2; do
for p in 0 1; do CLOVER_F2_PROBE=$p timeout 300 python scripts/f2_probe.py 3840 >> gpurun_out/f2_probe.jsonl; done
done
cat gpurun_out/f2_probe.jsonl
