# A/B of the y-sweep L2 cache policy variants (build_ab/, see CLOVER_L2HINT)
# Variants: python -c "from paper_conf_cluster_regulymg15_b200 import build as b; b.build(out='build_ab/libclover_h2.so', defines=('CLOVER_L2HINT=2',))" (and h1)
CLOVER_LIB=build_ab/libclover_h2.so timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "fused_y or bm64 or ragged" 2>&1 | tail -1
run() { CLOVER_LIB=$2 python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e --no-active | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['ms_per_step'],4), *[round(v['avg_ms'],4) for v in d['kernels'].values()], d['clocks']['reasons'])"; }
for i in 1 2; do
run h0 paper_conf_cluster_regulymg15_b200/libclover.so
run h1 build_ab/libclover_h1.so
run h2 build_ab/libclover_h2.so
done
