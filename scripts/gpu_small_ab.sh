# kernel_times on small meshes (960^2, 1920^2) and 3840^2 per variant (VARIANTS), two repeats
mkdir -p gpurun_out
: > gpurun_out/small_ab.txt
for r in 1 2; do
  for v in ${VARIANTS:-base}; do
    for n in 960 1920 3840; do
      t=$(CLOVER_LIB=build_ab/libclover_$v.so timeout 300 python scripts/kernel_times.py $n $n 40 2>/dev/null | python -c "import json,sys; print(round(json.loads(sys.stdin.read().strip().splitlines()[-1])['ms_per_step_graphs'],4))")
      echo "$v $n $r $t" >> gpurun_out/small_ab.txt
    done
  done
done
cat gpurun_out/small_ab.txt
