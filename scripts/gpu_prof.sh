set -x
mkdir -p gpurun_out
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"ks_" -s 30 -c 11 -o gpurun_out/prof_c3_r2 python scripts/prof_run.py 3840 3840 8 > gpurun_out/prof_c3_r2.log 2>&1
tail -2 gpurun_out/prof_c3_r2.log
