# One line per BASELINE config that fits one GPU (run under gpurun):
# C2 960^2 (87 steps), C4 7680^2 strong-scaling base at N=1.
mkdir -p gpurun_out
python bench.py --mesh 960 960 --steps 87 --warmup 5 --no-cpu-baseline --no-e2e --no-active > gpurun_out/c2.json 2>gpurun_out/c2.err
python bench.py --strong --steps 30 --warmup 5 --no-cpu-baseline --no-e2e --no-active > gpurun_out/c4.json 2>gpurun_out/c4.err
for f in c2 c4; do python -c "import json; d=json.loads(open('gpurun_out/$f.json').read().strip().splitlines()[-1]); print('$f', d['config']['mesh'], round(d['ms_per_step'],4), 'ms', round(d['value']/1e9,3), 'G/s', 'step_frac', round(d['roofline']['step_frac'],3))"; done
