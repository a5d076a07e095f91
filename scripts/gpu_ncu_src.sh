mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"ks_lagrangian|ks_advec_y|ks_visc|ks_advec_x" -s 200 -c 8 \
  -o gpurun_out/prof_src -f python scripts/prof_run.py 3840 3840 53 > gpurun_out/prof_src.log 2>&1
tail -2 gpurun_out/prof_src.log
