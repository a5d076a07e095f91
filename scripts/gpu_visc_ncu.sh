# ncu --set full of visc_dt (3 launches after step 50) for the default build and VSTG=8
mkdir -p gpurun_out
for v in base vstg8; do
  CLOVER_LIB=build_ab/libclover_$v.so timeout 900 ncu --set full --clock-control none -k regex:ks_visc -s 50 -c 3 \
    -o gpurun_out/visc_$v -f python scripts/prof_run.py 3840 3840 54 > gpurun_out/visc_$v.log 2>&1
done
ls -la gpurun_out
