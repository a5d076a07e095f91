# segment-chain A/B: kernel times (bm 3840^2 and active flow) per variant,
# DRAM bytes per kernel under ncu for base and chain0, then the GPU suite
mkdir -p gpurun_out
VARIANTS="${VARIANTS:-base chain0 chainp1 chainm1}" bash scripts/gpu_ks_ab.sh
cp gpurun_out/ks_ab.jsonl gpurun_out/chain_ab.jsonl
for v in base chain0; do
  CLOVER_LIB=build_ab/libclover_$v.so timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --clock-control none -k regex:ks_ -s 200 -c 12 --csv python scripts/prof_run.py 3840 3840 54 \
    > gpurun_out/chain_ncu_$v.csv 2> gpurun_out/chain_ncu_$v.err
done
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest.log
tail -3 gpurun_out/pytest.log
