for i in 1 2; do
python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('main', d['ms_per_step'], d['clocks'])"
CLOVER_LIB=build_ab/libclover_def.so python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('def ', d['ms_per_step'], d['clocks'])"
done
