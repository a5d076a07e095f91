# A/B with the fully-active-flow side measurement: bash scripts/ab_active.sh NAME...
for v in "$@"; do
  CLOVER_LIB=build_ab/libclover_$v.so python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['ms_per_step'],4), 'active', round(d['active_flow']['ms_per_step'],4))"
done
