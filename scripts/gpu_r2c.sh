mkdir -p gpurun_out
bash scripts/gpu_tests.sh
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 5 --warmup 3 --transport host > gpurun_out/bench_n2_host.json 2> gpurun_out/bench_n2_host.err
echo "n2 rc=$?"; tail -c 600 gpurun_out/bench_n2_host.json; tail -3 gpurun_out/bench_n2_host.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2>&1; echo "ref rc=$?"; tail -c 400 gpurun_out/bench_ref.json
