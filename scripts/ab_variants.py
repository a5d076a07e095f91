"""Build libclover variants with extra -D flags (CPU side) or time them on
the GPU (--run): python scripts/ab_variants.py [--run] NAME=DEF1,DEF2 ...
A definition list may include @GITREF to build that revision's sources."""
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
def build_ref(ref, path, defines):
    """Build the library from the sources of git revision `ref`."""
    import tempfile
    tmp = tempfile.mkdtemp()
    for rel in ("include/clover.h",) + tuple(
            "paper_conf_cluster_regulymg15_b200/csrc/" + f for f in
            subprocess.check_output(["git", "-C", ROOT, "ls-tree", "--name-only", ref,
                                     "paper_conf_cluster_regulymg15_b200/csrc/"], text=True).split()
            for f in [f.split("/")[-1]]):
        dst = os.path.join(tmp, rel)
        os.makedirs(os.path.dirname(dst), exist_ok=True)
        with open(dst, "w") as fh:
            fh.write(subprocess.check_output(["git", "-C", ROOT, "show", f"{ref}:{rel}"], text=True))
    cmd = [b.nvcc(), "-O3", "-std=c++17", b.ARCH, "-lineinfo", "-fmad=false", "-Xcompiler", "-fPIC",
           "-shared", "-I", os.path.join(tmp, "include"), "-o", path,
           os.path.join(tmp, "paper_conf_cluster_regulymg15_b200/csrc/clover_engine.cu")]
    cmd += ["-D" + d for d in defines]
    nd = b.nccl_dir()
    if nd:
        cmd += ["-DCLOVER_WITH_NCCL", "-I", os.path.join(nd, "include"), "-L", os.path.join(nd, "lib"),
                "-l:libnccl.so.2", "-Xlinker", "-rpath=" + os.path.join(nd, "lib")]
    subprocess.check_call(cmd)


for spec in specs:
    name, _, defs = spec.partition("=")
    path = os.path.join(outdir, f"libclover_{name}.so")
    if not run:
        dl = [d for d in defs.split(",") if d and not d.startswith("@")]
        refs = [d[1:] for d in defs.split(",") if d.startswith("@")]
        if refs:
            build_ref(refs[0], path, dl)
        else:
            b.build(out=path, defines=tuple(dl))
        print("built", path)
        continue
    env = dict(os.environ, CLOVER_LIB=path)
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "20", "--warmup", "3",
                          "--no-cpu-baseline", "--no-e2e", "--no-active", "--no-full"], env=env, capture_output=True, text=True)
    try:
        d = json.loads(out.stdout.strip().splitlines()[-1])
    except Exception:
        print(name, "FAILED", out.stderr[-2000:])
        continue
    ks = " ".join(f"{k.replace('k_advec_', '').replace('k_', '')}={v['avg_ms']:.3f}" for k, v in d["kernels"].items()
                  if v["avg_ms"] > 0.01)
    print(f"{name:14s} {d['ms_per_step']:.3f} ms/step  {ks}", flush=True)
