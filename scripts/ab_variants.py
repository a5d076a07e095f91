"""Build libclover variants with extra -D flags (CPU side) or time them on
the GPU (--run): python scripts/ab_variants.py [--run] NAME=DEF1,DEF2 ..."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cluster_regulymg15_b200 import build as b  # noqa: E402

run = "--run" in sys.argv
specs = [a for a in sys.argv[1:] if not a.startswith("--")]
outdir = os.path.join(ROOT, "build_ab")
os.makedirs(outdir, exist_ok=True)
for spec in specs:
    name, _, defs = spec.partition("=")
    path = os.path.join(outdir, f"libclover_{name}.so")
    if not run:
        b.build(out=path, defines=tuple(d for d in defs.split(",") if d))
        print("built", path)
        continue
    env = dict(os.environ, CLOVER_LIB=path)
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "20", "--warmup", "3",
                          "--no-cpu-baseline", "--no-e2e"], env=env, capture_output=True, text=True)
    try:
        d = json.loads(out.stdout.strip().splitlines()[-1])
    except Exception:
        print(name, "FAILED", out.stderr[-2000:])
        continue
    ks = " ".join(f"{k.replace('k_advec_', '').replace('k_', '')}={v['avg_ms']:.3f}" for k, v in d["kernels"].items()
                  if v["avg_ms"] > 0.01)
    print(f"{name:14s} {d['ms_per_step']:.3f} ms/step  {ks}", flush=True)
