# A/B kernel times over build_ab variants (VARIANTS), then the GPU suite on the default build
mkdir -p gpurun_out
VARIANTS="${VARIANTS:-base}" bash scripts/gpu_ks_ab.sh
cp gpurun_out/ks_ab.jsonl gpurun_out/var_ab.jsonl
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest.log
tail -3 gpurun_out/pytest.log
