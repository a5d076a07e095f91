# ncu --set full capture of one launch of each step kernel type (2 steps:
# x-first and y-first) into gpurun_out/prof_full.ncu-rep
mkdir -p gpurun_out
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"ks_" -s 25 -c 10 \
  -o gpurun_out/prof_full -f python scripts/prof_run.py 3840 3840 8 > gpurun_out/prof_full.log 2>&1
tail -2 gpurun_out/prof_full.log
