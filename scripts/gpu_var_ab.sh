# generic kernel_times A/B over build_ab/libclover_<variant>.so (VARIANTS), two repeats
mkdir -p gpurun_out
VARIANTS="${VARIANTS:-base}" bash scripts/gpu_ks_ab.sh
cp gpurun_out/ks_ab.jsonl gpurun_out/var_ab.jsonl
