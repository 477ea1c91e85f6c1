#!/usr/bin/env python
"""Stall-reason totals and the top stalled SASS lines of one kernel in an ncu report.

    python tools/ncu_stalls.py report.ncu-rep [kernel-regex] [--top N]
"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
kre = sys.argv[2] if len(sys.argv) > 2 and not sys.argv[2].startswith("--") else None
top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 12
args = ["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"]
if kre:
    args += ["-k", "regex:" + kre]
rows = list(csv.reader(io.StringIO(subprocess.run(args, capture_output=True, text=True).stdout)))
hdr, secs, cur = None, [], None
for r in rows:
    if r and r[0] == "Kernel Name":
        cur = []; secs.append((r[1], cur)); continue
    if r and r[0] == "Address":
        hdr = r; continue
    if hdr and cur is not None and len(r) == len(hdr):
        cur.append(dict(zip(hdr, r)))
for name, out in secs[:1]:
    cols = [c for c in hdr if c.startswith("stall_") and "Not Issued" not in c]
    tot = {c: sum(float(o[c] or 0) for o in out) for c in cols}
    T = sum(tot.values())
    print(name[:100])
    print("stall reasons:", ", ".join(f"{c[6:]} {v / T * 100:.1f}%" for c, v in sorted(tot.items(), key=lambda x: -x[1]) if v > T * 0.01))
    st = "Warp Stall Sampling (All Samples)"
    for i, o in sorted(enumerate(out), key=lambda x: -float(x[1][st] or 0))[:top]:
        t2 = sorted(((float(o[c] or 0), c[6:]) for c in cols), reverse=True)[:2]
        print(f"{i:5d} {float(o[st] or 0) / T * 100:5.1f}% {t2[0][1]}/{t2[1][1]} | {o['Source'][:90]}")
