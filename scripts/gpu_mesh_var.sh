# kernel_times graph step per variant (VARIANTS) on MESHES ("NX:NY ..."), two repeats
mkdir -p gpurun_out
: > gpurun_out/mesh_var.txt
for r in 1 2; do
  for v in ${VARIANTS:-base}; do
    for m in ${MESHES:-7680:960}; do
      nx=${m%:*}; ny=${m#*:}
      t=$(CLOVER_LIB=build_ab/libclover_$v.so timeout 300 python scripts/kernel_times.py $nx $ny 40 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step_graphs'],4), ' '.join(f'{k[2:]}={v:.4f}' for k,v in d['kernels_ms'].items() if v>0.005))")
      echo "$v $m $r $t" >> gpurun_out/mesh_var.txt
    done
  done
done
cat gpurun_out/mesh_var.txt
