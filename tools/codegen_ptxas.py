"""ptxas registers / spills of the generated A kernels (Table II analogue):
compiles csrc/gen/rhs_alg.cu for sm_100a with -Xptxas -v and tabulates."""
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CS = os.path.join(ROOT, "paper_conf_sc_fernandonhzsgb22_b200", "csrc")
cmd = ["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
       "-std=c++17", "-Xptxas", "-v", "-I", CS, "-I", os.path.join(ROOT, "include"), "-c",
       os.path.join(CS, "gen", "rhs_alg.cu"), "-o", "/tmp/rhs_alg.o"]
r = subprocess.run(cmd, capture_output=True, text=True)
txt = r.stdout + r.stderr
rows = []
for m in re.finditer(r"Compiling entry function '_ZN3dgr\d+(k_alg_\w+?)EPKd.*?\n.*?\n\s+(\d+) bytes stack frame, "
                     r"(\d+) bytes spill stores, (\d+) bytes spill loads\n.*?Used (\d+) registers", txt):
    rows.append(m.groups())
print("| kernel | registers | spill stores (B) | spill loads (B) | stack frame (B) |")
print("|---|---|---|---|---|")
for k, stack, st, ld, reg in sorted(rows):
    print(f"| {k} | {reg} | {st} | {ld} | {stack} |")
sys.exit(r.returncode)
