"""Static SASS size of each ks_* kernel of clover_engine.cu (instruction
count, and IMAD.MOV / LDS / fp64 counts): a quick CPU-side proxy for the
issue cost of a code change before spending GPU time.
python scripts/sass_count.py [-DFOO ...] [--filter NAME]"""
import collections
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
args = [a for a in sys.argv[1:] if not a.startswith("--filter")]
flt = next((a.split("=", 1)[1] for a in sys.argv[1:] if a.startswith("--filter=")), "ks_")
with tempfile.TemporaryDirectory() as td:
    cub = os.path.join(td, "e.cubin")
    subprocess.check_call(["nvcc", "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a",
                           "-fmad=false", "-I", os.path.join(ROOT, "include"), "-cubin", "-o", cub, *args,
                           os.path.join(ROOT, "paper_conf_cluster_regulymg15_b200/csrc/clover_engine.cu")])
    sass = subprocess.run(["cuobjdump", "-sass", cub], capture_output=True, text=True).stdout
fn, cnt = None, {}
for line in sass.splitlines():
    m = re.search(r"Function : (\S+)", line)
    if m:
        fn = m.group(1)
        cnt[fn] = collections.Counter()
        continue
    m = re.match(r"\s+/\*[0-9a-f]{4,}\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)", line)
    if fn and m:
        op = m.group(2)
        cnt[fn]["all"] += 1
        base = op.split(".")[0]
        if op.startswith("IMAD.MOV") or base == "MOV":
            cnt[fn]["mov"] += 1
        if base in ("DADD", "DMUL", "DFMA", "DSETP", "DMNMX"):
            cnt[fn]["fp64"] += 1
        if base == "LDS":
            cnt[fn]["lds"] += 1
        if base in ("BRA", "BSSY", "BSYNC"):
            cnt[fn]["br"] += 1
for fn, c in cnt.items():
    short = re.sub(r"_ZN6clover\d+", "", fn).split("E")[0]
    if flt in short or flt in fn:
        print(f"{short:28s} all {c['all']:6d} mov {c['mov']:5d} fp64 {c['fp64']:5d} lds {c['lds']:5d} br {c['br']:5d}")
