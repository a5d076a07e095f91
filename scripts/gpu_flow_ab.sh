mkdir -p gpurun_out; rm -f gpurun_out/flow_ab.jsonl
for i in 1 2; do for f in 0 1; do CLOVER_FLOW=$f timeout 120 python scripts/kernel_times.py 3840 3840 40 | sed "s/^{/{\"flow\": $f, /" >> gpurun_out/flow_ab.jsonl; done; done
python - <<'PY'
import json
for l in open('gpurun_out/flow_ab.jsonl'):
    d=json.loads(l); print(d["flow"], round(d["ms_per_step_graphs"],4), {k: round(v,4) for k,v in d["kernels_ms"].items()})
PY
