"""Collect the per-config bench lines of scripts/configs_run.sh
(gpurun_out/c2.json, c4.json) into profiles/<tag>_configs.json."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1] if len(sys.argv) > 1 else "r1"
out = {}
for f, name in (("c2", "configs[1] 960x960 bm, 87 steps"),
                ("c4", "configs[3] 7680x7680 bm, N=1 (strong-scaling base), 30 steps")):
    d = json.loads(open(os.path.join(ROOT, "gpurun_out", f + ".json")).read().strip().splitlines()[-1])
    out[name] = {"ms_per_step": d["ms_per_step"], "value": d["value"], "unit": d["unit"],
                 "steps": d["steps"], "step_frac": d["roofline"]["step_frac"],
                 "step_achieved_gbs": d["roofline"]["step_achieved"],
                 "kernels_ms": {k: v["avg_ms"] for k, v in d["kernels"].items()},
                 "clocks": d["clocks"]}
json.dump(out, open(os.path.join(ROOT, "profiles", tag + "_configs.json"), "w"), indent=1)
print(json.dumps({k: round(v["value"] / 1e9, 3) for k, v in out.items()}))
