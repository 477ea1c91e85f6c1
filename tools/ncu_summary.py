#!/usr/bin/env python
"""Summarise an ncu --set full report of the probe: key metrics + top SASS lines by stall samples.

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep [--json out.json] [--top 25]
"""
import argparse
import collections
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "lts__t_sectors_srcunit_tex_op_read.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
        "sm__cycles_elapsed.avg.per_second", "launch__grid_size", "launch__block_size",
        "l1tex__t_sector_hit_rate.pct", "lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum",
        "smsp__sass_inst_executed_op_shared_ld.sum", "smsp__sass_inst_executed_op_shared_atom.sum",
        "smsp__sass_inst_executed_op_global_ld.sum", "smsp__sass_inst_executed_op_global_st.sum",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "smsp__inst_executed_op_branch.sum"]


def ncu(rep, *args):
    return subprocess.run(["ncu", "-i", rep, *args], capture_output=True, text=True).stdout


def raw(rep):
    rows = list(csv.reader(io.StringIO(ncu(rep, "--page", "raw", "--csv"))))
    h, u, v = rows[0], rows[1], rows[2]
    out = {}
    for i, n in enumerate(h):
        if n.startswith("smsp__pcsamp_warps_issue_stalled_") and not n.endswith("_not_issued"):
            try:
                val = float(v[i].replace(",", ""))
            except ValueError:
                continue
            if val > 0:
                out.setdefault("stall_samples_by_reason", {})[n.replace("smsp__pcsamp_warps_issue_stalled_", "")] = val
            continue
        if n in KEYS:
            try:
                out[n] = {"value": float(v[i].replace(",", "")), "unit": u[i]}
            except ValueError:
                out[n] = {"value": v[i], "unit": u[i]}
    return out


def source(rep, top):
    rows = list(csv.reader(io.StringIO(ncu(rep, "--page", "source", "--csv", "--print-source", "sass"))))
    secs, cur = [], None
    for r in rows:
        if r and r[0] == "Kernel Name":
            cur = {"name": r[1], "rows": []}; secs.append(cur); continue
        if r and r[0] == "Address":
            cur["hdr"] = r; continue
        if cur is not None and r:
            cur["rows"].append(r)
    res = []
    for s in secs:
        h = s["hdr"]; si = h.index("Warp Stall Sampling (All Samples)"); ie = h.index("Instructions Executed")
        src = h.index("Source")
        tot_s = sum(float(r[si] or 0) for r in s["rows"]); tot_i = sum(float(r[ie] or 0) for r in s["rows"])
        ops = collections.Counter()
        for r in s["rows"]:
            t = r[src].split()
            op = t[1] if t and t[0].startswith("@") else (t[0] if t else "?")
            ops[op] += float(r[si] or 0)
        res.append({"function": s["name"][:120], "stall_samples": tot_s, "inst_executed": tot_i,
                    "top_ops_by_stall": ops.most_common(top)})
    return res


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--json")
    ap.add_argument("--top", type=int, default=15)
    a = ap.parse_args()
    d = {"report": a.rep, "metrics": raw(a.rep), "functions": source(a.rep, a.top)}
    s = json.dumps(d, indent=1)
    if a.json:
        open(a.json, "w").write(s)
    print(s)
