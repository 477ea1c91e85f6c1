#!/usr/bin/env python
"""Compile one .cu for sm_100a with -Xptxas -v and print registers / spills per kernel.

    python tools/ptxas_report.py paper_conf_icde_doraiswamyf22_b200/csrc/probe.cu [filter]
"""
import re
import subprocess
import sys

src = sys.argv[1]
flt = sys.argv[2] if len(sys.argv) > 2 else ""
r = subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
                    "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC", "-Xptxas", "-v", "-Iinclude",
                    "-dc", "-o", "/tmp/_ptxas_report.o", src], capture_output=True, text=True)
if r.returncode:
    print(r.stderr)
    sys.exit(1)
cur = None
for line in r.stderr.splitlines():
    m = re.search(r"Compiling entry function '([^']+)'", line)
    if m:
        name = m.group(1)
        d = re.search(r"(k_\w+?)I(L.*?)EE", name)
        cur = (d.group(1) + "<" + ",".join(re.findall(r"Li(\d+)E?", d.group(2))) + ">") if d else name[-60:]
        continue
    if cur and "spill" in line:
        sp = re.search(r"(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads", line)
        stack, st, ld = sp.groups()
    if cur and "Used" in line and "registers" in line:
        regs = re.search(r"Used (\d+) registers", line).group(1)
        smem = re.search(r"(\d+) bytes smem", line)
        if flt in cur:
            print(f"{cur:28s} regs {regs:>3s}  stack {stack:>4s}  spill st/ld {st}/{ld}  smem {smem.group(1) if smem else 0}")
        cur = None
