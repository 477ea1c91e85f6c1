#!/usr/bin/env python
"""Per-CUDA-source-line stall samples and instruction shares of an ncu --set full report (needs
-lineinfo):  python tools/ncu_lines.py gpurun_out/x.ncu-rep [--top 25]"""
import argparse
import csv
import io
import subprocess

ap = argparse.ArgumentParser()
ap.add_argument("rep")
ap.add_argument("--top", type=int, default=25)
a = ap.parse_args()
txt = subprocess.run(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
fn, hdr, out = None, None, []
for r in csv.reader(io.StringIO(txt)):
    if not r:
        continue
    if r[0] == "Function Name":
        fn = r[1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr and r[0] and r[0] != "File Path":
        try:
            line = int(r[0])
            d = dict(zip(hdr, r))
            s = float(d["Warp Stall Sampling (All Samples)"] or 0)
            ie = float(d["Instructions Executed"] or 0)
        except (ValueError, KeyError):
            continue
        out.append((s, ie, fn.split("(")[0].split("::")[-1], line, r[1].strip()[:110]))
ts, ti = sum(o[0] for o in out) or 1, sum(o[1] for o in out) or 1
print(f"{'stall%':>6} {'inst%':>6}  function:line  source")
for o in sorted(out, reverse=True)[:a.top]:
    print(f"{100 * o[0] / ts:6.1f} {100 * o[1] / ti:6.1f}  {o[2]}:{o[3]}  {o[4]}")
