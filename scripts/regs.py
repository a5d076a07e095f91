"""Print registers / spills per kernel of clover_engine.cu for extra -D flags:
python scripts/regs.py [-DFOO ...]"""
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
out = subprocess.run(["nvcc", "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-fmad=false",
                      "-I", os.path.join(ROOT, "include"), "-Xptxas", "-v", "-c", "-o", "/dev/null",
                      *sys.argv[1:], os.path.join(ROOT, "paper_conf_cluster_regulymg15_b200/csrc/clover_engine.cu")],
                     capture_output=True, text=True).stderr
name = None
for line in out.splitlines():
    m = re.search(r"Compiling entry function '_ZN6clover\d+(ks_\w+?)(ILi(\d)EE)?E", line)
    if m:
        name = m.group(1) + (f"<{m.group(3)}>" if m.group(3) else "")
        continue
    if name and "spill" in line:
        sp = re.findall(r"(\d+) bytes spill", line)
    if name and "Used" in line:
        print(f"{name:22s} regs {re.search(r'Used (\d+)', line).group(1):>4s} spill st/ld {sp}")
        name = None
