# full 300-step configs[2] run (bench full_run, median of 3 fresh contexts) per variant, two rounds
mkdir -p gpurun_out
: > gpurun_out/full_ab.txt
for r in 1 2; do
  for v in ${VARIANTS:-base}; do
    CLOVER_LIB=build_ab/libclover_$v.so timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-active > gpurun_out/full_$v.json 2>/dev/null
    python -c "import json; d=json.loads(open('gpurun_out/full_$v.json').read().strip().splitlines()[-1]); print('$v', $r, round(d['ms_per_step'],4), round(d['full_run']['ms_per_step'],4))" >> gpurun_out/full_ab.txt
  done
done
cat gpurun_out/full_ab.txt
