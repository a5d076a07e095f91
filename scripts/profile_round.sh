# Round profiling bundle (run under gpurun; writes gpurun_out/, then
# scripts/summarize_profiles.py copies the summaries into profiles/).
set -x
mkdir -p gpurun_out
# 1) the bench line itself (no profiler)
python bench.py --steps 50 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err
tail -1 gpurun_out/bench.json | head -c 600; echo
# 2) launch list of the same command (cold-cache, serialised per-launch times)
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_under_ncu.log 2>&1
# 3) full capture of every step kernel type (2 steps: x-first and y-first)
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"ks_" -s 25 -c 10 \
  -o gpurun_out/prof_full python scripts/prof_run.py 3840 3840 8 > gpurun_out/prof_full.log 2>&1
ls -la gpurun_out
