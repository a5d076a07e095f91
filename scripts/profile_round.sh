# Round profiling bundle (run under gpurun; writes gpurun_out/, then
# `python scripts/summarize_profiles.py <tag>` copies the summaries into profiles/).
set -x
mkdir -p gpurun_out
# 1) the bench line itself (no profiler)
python bench.py --steps 50 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err
tail -1 gpurun_out/bench.json | head -c 600; echo
# 2) launch list of the same command (cold-cache, serialised per-launch times)
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-full --no-active > gpurun_out/bench_under_ncu.log 2>&1
# 3) full capture of every step kernel type, 3 steps (x-first, y-first,
#    x-first) after step 50 (4 streaming ks_ kernels per step: skip 4*50)
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"ks_" -s 200 -c 12 \
  -o gpurun_out/prof_full -f python scripts/prof_run.py 3840 3840 54 > gpurun_out/prof_full.log 2>&1
# 4) NCCL kernels in the virtual-remote NCCL mode (launch list)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_nccl.csv python scripts/prof_nccl.py > gpurun_out/prof_nccl.log 2>&1
ls -la gpurun_out
