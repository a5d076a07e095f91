# A/B of programmatic dependent launch on the streaming (CLOVER_PDL) and the
# fixup launches (CLOVER_PDL_FIX) at the other configs; variants built by
# scripts/ab_variants.py p11= p00=CLOVER_PDL=0,CLOVER_PDL_FIX=0 p01=CLOVER_PDL=0,CLOVER_PDL_FIX=1
run() { CLOVER_LIB=build_ab/libclover_$1.so python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e --no-active $2 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', d['config']['mesh'], round(d['ms_per_step'],4), d['clocks']['reasons'])"; }
for i in 1 2; do for v in p11 p00 p01; do run $v "--mesh 960 960"; run $v --strong; done; done
