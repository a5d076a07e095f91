# A/B of the y-wall band fold (run under gpurun).  Build the reference variant first:
#   python -c "from paper_conf_cluster_regulymg15_b200 import build as b; b.build(out='build_ab/libclover_old.so', defines=('CLOVER_YWALLS_FOLD=0',))"
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -2; CLOVER_LIB=build_ab/libclover_old.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -1
for i in 1 2 3; do
python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('new', d['ms_per_step'], *[round(v['avg_ms'],4) for v in d['kernels'].values()], d['gpu_launches'], d['clocks']['reasons'])"
CLOVER_LIB=build_ab/libclover_old.so python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('old', d['ms_per_step'], *[round(v['avg_ms'],4) for v in d['kernels'].values()], d['gpu_launches'], d['clocks']['reasons'])"
done
