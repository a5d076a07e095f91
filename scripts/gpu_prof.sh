set -x
mkdir -p gpurun_out
./scripts/fp64_peak > gpurun_out/fp64_peak.jsonl 2>&1; cat gpurun_out/fp64_peak.jsonl
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches.csv python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_under_ncu.log 2>&1
tail -2 gpurun_out/launches.csv
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_visc_dt|k_lagrangian|k_advec" -s 30 -c 12 -o gpurun_out/prof_c3 python scripts/prof_run.py 3840 3840 8 > gpurun_out/prof_c3.log 2>&1
tail -3 gpurun_out/prof_c3.log
ls -la gpurun_out
