set -x
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('value',d['value']/1e9,'G  ms/step',d['ms_per_step'],'step_frac',d['roofline']['step_frac']); 
[print(f'{k:22s} {v[\"avg_ms\"]:.3f} ms  {v[\"achieved_gbs\"] or 0:7.0f} GB/s') for k,v in d['kernels'].items()]; print('e2e', d['e2e'])"
