#!/usr/bin/env python
"""bench.py — points/s of the point-polygon join + COUNT on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload c3|c5] [--impl spade|reference]

One step = one pass of the whole hot path over one batch of synthetic input resident in HBM:
spade_join_count over this GPU's shard of points (canvas lookup + exact boundary tests + COUNT
aggregation, Sec. 5.2) and, for N > 1, the NCCL all-reduce of the int64 counts.
Default workload: config 3 of BASELINE.json (1B taxi-like points per GPU x 260 neighbourhood-like
polygons); N GPUs process N x 1B points (weak scaling, canvas replicated).  Inputs are 8 GB per GPU,
far larger than the 126 MB L2, so no L2 flush is needed between steps.

Prints ONE JSON line on rank 0.  --impl reference times the CPU
oracle (the only reference this paper-only task has) on a bounded sample, on the host cores.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "points/sec for point-polygon join+COUNT at 1/2/4/8 B200; HBM GB/s vs peak"
FALLBACK_HBM_GBS = 6650.0


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--workload", default="c3", choices=["c1", "c2", "c3", "c4", "c5", "dj", "dj2", "knn", "ov", "pp"],
                    help="c3 (default) = the metric's join+COUNT config; c2 select, c4 pairs, c5 40k polygons; "
                         "dj / dj2 distance joins (type 1 pairs / type 2 count), knn kNN selection, "
                         "ov overlap-heavy polygon set (1,000 overlapping stars), pp polygon x polygon join")
    ap.add_argument("--points-per-gpu", type=int, default=None, help="default: the config's size (1B; C2 100M)")
    ap.add_argument("--impl", default="spade", choices=["spade", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-parity", action="store_true", help="skip the oracle parity check on the sample")
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="target CPU oracle sample time")
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no e2e/cpu/clocks)")
    ap.add_argument("--dense", action="store_true", help="force the dense fine-canvas layout (A/B runs)")
    ap.add_argument("--count", action="store_true", help="run COUNT on the workload's canvas and points (A/B of the sinks)")
    ap.add_argument("--layers", action="store_true",
                    help="COUNT through the paper's layer index (spade_build_layered: one probe pass per layer of "
                         "non-intersecting polygons) instead of the owner sets of one canvas (A/B, P:148 / P:270-274)")
    ap.add_argument("--max-dim", type=int, default=None, help="override the workload's canvas max_dim")
    ap.add_argument("--opt", action="append", default=[], metavar="NAME=VALUE",
                    help="spade_set_option before the run (A/B of probe paths; results never depend on it)")
    return ap.parse_args()


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


METRICS = {
    "count": METRIC,
    "select": "points/sec for spatial selection (ids of points inside the query polygon)",
    "pairs": "points/sec for point-polygon join emitting (point_id, polygon_id) pairs",
    "dist_pairs": "points/sec for the type 1 distance join emitting (point_id, disk_id) pairs",
    "dist_count": "points/sec for the type 2 distance join COUNT (per-disk counts)",
    "knn": "points/sec scanned by kNN selection (circle aggregation + distance select + sort)",
    "polyjoin": "polygon pairs/sec decided by the polygon x polygon join (|D1| x |D2| per call)",
}


def workload(name, n_per_gpu):
    from gen import configs
    if name in configs.POLYJOIN:
        return configs.POLYJOIN[name]()
    if name in configs.DISTANCE:
        return configs.DISTANCE[name](n_per_gpu or 1_000_000_000)
    if name in ("c1", "c2"):
        return getattr(configs, name)() if n_per_gpu is None else getattr(configs, name)(n_per_gpu)
    return getattr(configs, name)(n_per_gpu or 1_000_000_000)


def measured_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def ncu_traffic(workload_name):
    """DRAM bytes per probe launch from the committed ncu --set full summary, if present."""
    p = os.path.join(ROOT, "profiles", "probe_ncu_summary.json")
    try:
        with open(p) as f:
            d = json.load(f)
        e = d.get(workload_name) or {}
        return e.get("dram_bytes_per_launch"), e.get("source")
    except Exception:
        return None, None


class ClockSampler:
    """NVML sampling of SM clock + throttle reasons during the timed region."""

    def __init__(self, index):
        self.index, self.samples, self.reasons, self.max_mhz = index, [], set(), None
        self._stop = threading.Event()
        self._t = None

    def start(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
            names = {
                getattr(nv, "nvmlClocksEventReasonHwSlowdown", 0x8): "hw_slowdown",
                getattr(nv, "nvmlClocksEventReasonHwThermalSlowdown", 0x40): "hw_thermal_slowdown",
                getattr(nv, "nvmlClocksEventReasonSwThermalSlowdown", 0x20): "sw_thermal_slowdown",
                getattr(nv, "nvmlClocksEventReasonSwPowerCap", 0x4): "sw_power_cap",
                getattr(nv, "nvmlClocksEventReasonHwPowerBrakeSlowdown", 0x80): "hw_power_brake",
            }

            def run():
                while not self._stop.is_set():
                    try:
                        self.samples.append(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM))
                        r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                        for bit, nm in names.items():
                            if r & bit:
                                self.reasons.add(nm)
                    except Exception:
                        pass
                    time.sleep(0.005)
            self._t = threading.Thread(target=run, daemon=True)
            self._t.start()
        except Exception as e:  # NVML missing: report nothing rather than invent
            self.error = str(e)

    def stop(self):
        self._stop.set()
        if self._t:
            self._t.join()
        med = statistics.median(self.samples) if self.samples else None
        return {"sm_mhz": med, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(self.samples)}


def _oracle_run(w, xy, nt):
    """The oracle call matching the workload's operation (as it stands)."""
    import numpy as np
    import oracle
    if getattr(w, "op", "") == "knn":
        oracle.knn(xy, w.query, w.k)
        return np.zeros(1, np.int64)
    if hasattr(w, "disks"):
        return oracle.disk_join_count(xy, w.disks, nthreads=nt)
    return oracle.join_count(xy, w.polys, nthreads=nt)


def cpu_oracle_rate(w, target_s, seed_offset=0):
    """Time the oracle (as it stands) on a bounded sample of the workload's points."""
    import numpy as np
    import gen
    import oracle
    nt = oracle.default_threads()
    if hasattr(w, "disks"):
        idx = np.arange(0, 2000, dtype=np.int64) * 499 + seed_offset
        pilot = gen.points_at(w.points, w.point_seed, idx)
        t0 = time.perf_counter()
        _oracle_run(w, pilot, nt)
        dt = max(time.perf_counter() - t0, 1e-3)
        m = int(max(2000, min(50_000_000, len(pilot) * target_s / dt)))
        stride = max(1, w.n_points // m)
        xy = gen.points_at(w.points, w.point_seed, np.arange(m, dtype=np.int64) * stride + seed_offset)
        t0 = time.perf_counter()
        counts = _oracle_run(w, xy, nt)
        dt = time.perf_counter() - t0
        what = (f"kNN (k={w.k}) by sorting all sampled points" if w.op == "knn" else
                f"x {len(w.disks['r2'])} disks, brute force over all pairs")
        return {"value": m / dt, "unit": "points/s", "cores": 1 if w.op == "knn" else nt, "kind": "oracle",
                "sample": f"{m} points = every {stride}-th global index of the workload's point stream, {what} "
                          f"({dt:.1f} s)", "seconds": dt, "sum_counts": 0,
                "idx": np.arange(m, dtype=np.int64) * stride + seed_offset, "rate": m / dt,
                "counts": None if w.op == "knn" else counts}
    idx = np.arange(0, 2000, dtype=np.int64) * 499 + seed_offset
    pilot = gen.points_at(w.points, w.point_seed, idx)
    t0 = time.perf_counter()
    oracle.join_count(pilot, w.polys, nthreads=nt)
    dt = max(time.perf_counter() - t0, 1e-3)
    m = int(max(2000, min(5_000_000, len(pilot) * target_s / dt)))
    stride = max(1, w.n_points // m)
    idx = np.arange(m, dtype=np.int64) * stride + seed_offset
    xy = gen.points_at(w.points, w.point_seed, idx)
    t0 = time.perf_counter()
    counts = oracle.join_count(xy, w.polys, nthreads=nt)
    dt = time.perf_counter() - t0
    return {"value": m / dt, "unit": "points/s", "cores": nt, "kind": "oracle",
            "sample": f"{m} points = every {stride}-th global index of the workload's point stream, "
                      f"x {len(w.polys['poly_ring_off']) - 1} polygons, brute force over all pairs "
                      f"({dt:.1f} s)", "seconds": dt, "sum_counts": int(counts.sum()),
            "idx": idx, "counts": counts, "rate": m / dt}


def cpu_rtree_rate(w, target_s):
    """The simple R-tree CPU join (STR over polygon bboxes + exact predicate), as it stands, on an
    index-strided sample of the workload's points, all host cores."""
    import numpy as np
    import gen
    import oracle
    nt = oracle.default_threads()
    pilot = gen.points_at(w.points, w.point_seed, np.arange(0, 20000, dtype=np.int64) * 4999)
    t0 = time.perf_counter()
    oracle.rtree_join_count(pilot, w.polys, nthreads=nt)
    dt = max(time.perf_counter() - t0, 1e-3)
    m = int(max(20000, min(50_000_000, len(pilot) * target_s / dt)))
    stride = max(1, w.n_points // m)
    xy = gen.points_at(w.points, w.point_seed, np.arange(m, dtype=np.int64) * stride)
    t0 = time.perf_counter()
    oracle.rtree_join_count(xy, w.polys, nthreads=nt)
    dt = time.perf_counter() - t0
    return {"value": m / dt, "unit": "points/s", "cores": nt, "kind": "rtree",
            "sample": f"{m} points = every {stride}-th global index, STR R-tree over "
                      f"{len(w.polys['poly_ring_off']) - 1} polygon bboxes + exact predicate ({dt:.1f} s)"}


def parity_check(w, cv, sp, idx, oracle_counts=None, rate=None, pairs_seconds=5.0):
    """The GPU path on the oracle's sample ("the GPU is run on the same
    subsample indices for parity"): per-polygon counts of the whole sample (the oracle's, from
    the timed cpu_baseline run when given) and the sorted (point, polygon) pairs of a prefix sized
    to ~pairs_seconds of oracle time, bit-exact.  Inputs regenerated from the shared seeded
    generator; expected values only from oracle/."""
    import numpy as np
    import torch
    import gen
    import oracle
    xy = gen.points_at(w.points, w.point_seed, idx)
    xy_d = torch.as_tensor(xy).cuda()
    res = {"sample": int(len(idx)), "indices": f"global indices {int(idx[0])}, {int(idx[1]) if len(idx) > 1 else ''}, ... "
                                                 f"(stride {int(idx[1] - idx[0]) if len(idx) > 1 else 0})"}
    if getattr(w, "op", "") == "knn":
        xy, xy_d = xy[:2_000_000], xy_d[:2_000_000]
        res["sample"] = int(len(xy))
        k = min(w.k, len(xy))
        gi, gd = sp.knn(xy_d, w.query, k)
        oi, od = oracle.knn(xy, w.query, k)
        res.update({"checked": f"kNN (k={k}) of the sample: ids and squared distances in order",
                    "ok": bool(np.array_equal(gi.cpu().numpy(), oi) and np.array_equal(gd.cpu().numpy(), od))})
        return res
    is_dist = hasattr(w, "disks")
    count_o = (lambda x: oracle.disk_join_count(x, w.disks)) if is_dist else (lambda x: oracle.join_count(x, w.polys))
    pairs_o = (lambda x: oracle.disk_join_pairs(x, w.disks)) if is_dist else (lambda x: oracle.join_pairs(x, w.polys))
    if oracle_counts is None:
        oracle_counts = count_o(xy)
    gc = sp.join_count(cv, xy_d).cpu().numpy()
    counts_ok = bool(np.array_equal(gc, oracle_counts))
    kp = len(idx) if rate is None else int(max(200, min(len(idx), rate * pairs_seconds)))
    opt, opl = pairs_o(xy[:kp])
    cap = int(sp.join_count(cv, xy_d[:kp]).sum())
    gpt, gpl = sp.join_pairs(cv, xy_d[:kp], capacity=max(cap, 1))
    gpt, gpl = gpt.cpu().numpy().astype(np.int64), gpl.cpu().numpy().astype(np.int64)
    o = np.lexsort((gpl, gpt))
    pairs_ok = bool(np.array_equal(gpt[o], opt) and np.array_equal(gpl[o], opl))
    res.update({"checked": f"per-{'disk' if is_dist else 'polygon'} COUNT of all {len(idx)} sample points; "
                           f"sorted (point, {'disk' if is_dist else 'polygon'}) pairs of the first {kp}",
                "counts_equal": counts_ok, "pairs_sample": kp, "pairs": int(len(opt)), "pairs_equal": pairs_ok,
                "ok": counts_ok and pairs_ok})
    return res


def polyjoin_oracle_rate(w, target_s, offset=0):
    """The polygon x polygon oracle (brute force over every polygon pair and edge pair) on the
    first k polygons of D1 (rotated by `offset`) x all of D2, k sized to ~target_s."""
    import oracle
    n1, n2 = len(w.polys["poly_ring_off"]) - 1, len(w.polys2["poly_ring_off"]) - 1

    def subset(k):
        import numpy as np
        pro = np.asarray(w.polys["poly_ring_off"])
        ro = np.asarray(w.polys["ring_off"])
        lo = offset % max(1, n1 - k)
        r0, r1 = pro[lo], pro[lo + k]
        v0, v1 = ro[r0], ro[r1]
        return {"ring_xy": np.asarray(w.polys["ring_xy"])[v0:v1], "ring_off": ro[r0:r1 + 1] - v0,
                "poly_ring_off": pro[lo:lo + k + 1] - r0}, lo
    sub, _ = subset(4)
    t0 = time.perf_counter()
    oracle.polygon_join(sub, w.polys2)
    dt = max(time.perf_counter() - t0, 1e-3)
    k = int(max(4, min(n1, 4 * target_s / dt)))
    sub, lo = subset(k)
    t0 = time.perf_counter()
    a, b = oracle.polygon_join(sub, w.polys2)
    dt = time.perf_counter() - t0
    return {"value": k * n2 / dt, "unit": "polygon pairs/s", "cores": oracle.default_threads(), "kind": "oracle",
            "sample": f"D1 polygons [{lo}, {lo + k}) x all {n2} of D2, brute force over every polygon and edge pair "
                      f"({dt:.1f} s)", "seconds": dt, "subset": sub, "lo": lo, "pairs": (a + lo, b)}


def run_reference(a):
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    w = workload(a.workload, a.points_per_gpu)
    if w.op == "polyjoin":
        per_step = max(1.0, 120.0 / max(1, a.steps + a.warmup))
        rates, secs, res = [], 0.0, None
        for k in range(a.steps):
            res = polyjoin_oracle_rate(w, per_step, offset=97 * k)
            rates.append(res["value"])
            secs += res["seconds"]
        value = statistics.median(rates)
        print(json.dumps({"impl": "reference", "metric": METRICS["polyjoin"], "value": value, "unit": "polygon pairs/s",
                          "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup, "ms_per_step": 1e3 * secs / max(1, a.steps),
                          "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int64",
                          "data": "synthetic", "config": {"workload": w.name, "desc": w.desc},
                          "cpu_baseline": {"value": value, "unit": "polygon pairs/s", "cores": res["cores"], "kind": "oracle",
                                           "sample": res["sample"]},
                          "e2e": {"value": value, "unit": "polygon pairs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}),
              flush=True)
        return
    per_step = max(1.0, 120.0 / max(1, a.steps + a.warmup))
    res = None
    for _ in range(a.warmup):
        cpu_oracle_rate(w, per_step / 8)
    rates, secs = [], 0.0
    for k in range(a.steps):
        res = cpu_oracle_rate(w, per_step, seed_offset=k)
        rates.append(res["value"])
        secs += res["seconds"]
    value = statistics.median(rates)
    op = w.op
    is_dist = hasattr(w, "disks")
    line = {
        "impl": "reference", "metric": METRICS[("dist_" + op) if is_dist and op != "knn" else op], "value": value, "unit": "points/s", "n_gpus": a.gpus,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": 1e3 * secs / max(1, a.steps),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int64",
        "data": "synthetic", "config": {"workload": w.name, "desc": w.desc, "points_per_gpu": w.n_points},
        "cpu_baseline": {"value": value, "unit": "points/s", "cores": res["cores"], "kind": "oracle",
                         "sample": res["sample"]},
        "e2e": {"value": value, "unit": "points/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "note": "reference arm = the CPU oracle (brute-force half-open even-odd PIP, __int128), "
                "on a bounded index-strided sample per step; the paper ships no code",
    }
    print(json.dumps(line), flush=True)


def run_polyjoin(a, w, sp, ws, rank, local):
    """Polygon x polygon join (spade_join_polygons): one step = one whole join call (both canvases
    built on a common grid, contact tests, ring-vertex probes, sort + unique) over device-resident
    polygon arrays; e2e = the same call from host (numpy) arrays, H2D inside the timing."""
    import numpy as np
    import torch
    import torch.distributed as dist
    dev = torch.device("cuda", local)
    n1, n2 = len(w.polys["poly_ring_off"]) - 1, len(w.polys2["poly_ring_off"]) - 1
    dA = {k: torch.as_tensor(np.ascontiguousarray(v)).to(dev) for k, v in w.polys.items()}
    dB = {k: torch.as_tensor(np.ascontiguousarray(v)).to(dev) for k, v in w.polys2.items()}
    stream = torch.cuda.current_stream()
    res = [None]

    def step():
        res[0] = sp.join_polygons(dA, dB, max_dim=w.max_dim)
    for _ in range(max(3, a.warmup)):
        step()
    torch.cuda.synchronize()
    sampler = ClockSampler(local)
    if not a.profile:
        sampler.start()
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    l0 = sp.launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(a.steps):
        step()
    e1.record(stream)
    torch.cuda.synchronize()
    l1 = sp.launch_count()
    clocks = sampler.stop() if not a.profile else None
    t_ms = e0.elapsed_time(e1)
    if ws > 1:
        tt = torch.tensor([t_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_ms = tt.item()
    ga, gb = (x.cpu().numpy().astype(np.int64) for x in res[0])
    value = ws * n1 * n2 * a.steps / (t_ms / 1e3)
    line = None
    if rank == 0:
        V = int(len(w.polys["ring_xy"]) + len(w.polys2["ring_xy"]))
        ms = t_ms / a.steps
        line = {"metric": METRICS["polyjoin"], "value": value, "unit": "polygon pairs/s", "n_gpus": ws, "steps": a.steps,
                "warmup": max(3, a.warmup), "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
                "vs_baseline": None, "dtype": "int32", "data": "synthetic",
                "config": {"workload": w.name, "desc": w.desc, "polygons": [n1, n2], "vertices": V, "max_dim": w.max_dim,
                           "parallelism": f"dp{ws} (replicated join per rank)",
                           "l2": "one whole join per step (two canvas builds, contact tests, probes, sort)"},
                "roofline": {"bound": "latency", "achieved": 16.0 * V / (ms / 1e3) / 1e9, "peak": measured_peak()[0],
                             "unit": "GB/s", "frac": 16.0 * V / (ms / 1e3) / 1e9 / measured_peak()[0], "traffic": None,
                             "kernel": "spade_join_polygons (whole call: builds + k_pp_contacts + probes + sort)",
                             "note": "algorithmic bytes = 16 B per input vertex (read by each of the two builds); "
                                     "the call is a chain of small kernels and host syncs: latency-bound"},
                "gpu_launches": int(l1 - l0), "check": {"pairs": int(len(ga))}}
        if clocks:
            line["clocks"] = clocks
        if not a.no_e2e and not a.profile:
            times = []
            for _ in range(a.e2e_steps):
                torch.cuda.synchronize()
                s0 = time.perf_counter()
                r = sp.join_polygons(w.polys, w.polys2, max_dim=w.max_dim)
                r[0].cpu()
                times.append(time.perf_counter() - s0)
            line["e2e"] = {"value": n1 * n2 / statistics.median(times), "unit": "polygon pairs/s",
                           "h2d_bytes_per_step": int(sum(np.asarray(v).nbytes for d in (w.polys, w.polys2) for v in d.values())),
                           "d2h_bytes_per_step": int(8 * len(ga)), "api": "join_polygons from host numpy arrays",
                           "timing": "host wall clock around the call"}
        if not a.no_cpu_baseline and not a.profile and ws == 1:
            cb = polyjoin_oracle_rate(w, a.cpu_seconds)
            sub, lo, (oa, ob) = cb.pop("subset"), cb.pop("lo"), cb.pop("pairs")
            cb.pop("seconds")
            line["cpu_baseline"] = cb
            if not a.no_parity:
                sa, sb = (x.cpu().numpy().astype(np.int64) for x in sp.join_polygons(sub, w.polys2, max_dim=w.max_dim))
                m = (ga >= lo) & (ga < lo + len(sub["poly_ring_off"]) - 1)
                line["parity"] = {"sample": f"D1 polygons [{lo}, {lo + len(sub['poly_ring_off']) - 1}) x all of D2",
                                  "checked": "sorted (a, b) pairs of the sample: oracle vs GPU on the sample, and vs "
                                             "the full GPU join restricted to the sample",
                                  "pairs": int(len(oa)),
                                  "ok": bool(np.array_equal(sa + lo, oa) and np.array_equal(sb, ob) and
                                             np.array_equal(ga[m], oa) and np.array_equal(gb[m], ob))}
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()


def main():
    a = parse()
    if a.impl == "reference":
        return run_reference(a)
    import numpy as np
    import torch
    import torch.distributed as dist

    import gen
    import paper_conf_icde_doraiswamyf22_b200 as sp

    ws, rank, local = dist_env()
    if ws != a.gpus and rank == 0:
        print(f"warning: --gpus {a.gpus} but WORLD_SIZE {ws}", file=sys.stderr)
    # one process per GPU; SPADE_DIST_BACKEND=gloo lets several ranks share one GPU (a test of the
    # multi-rank flow on a 1-GPU box: device = local rank modulo the device count)
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    if ws > 1:
        backend = os.environ.get("SPADE_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    sp.load()
    for o in a.opt:
        k, v = o.split("=")
        sp.set_option(k, int(v))
    w = workload(a.workload, a.points_per_gpu)
    if w.op == "polyjoin":
        return run_polyjoin(a, w, sp, ws, rank, local)
    if a.count and w.op in ("select", "pairs"):
        w.op = "count"
    n = w.n_points
    is_dist = hasattr(w, "disks")
    P = len(w.disks["r2"]) if is_dist else len(w.polys["poly_ring_off"]) - 1
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream()

    # canvas build (timed separately; not part of a step); kNN builds no canvas (knn.cu).  Built
    # twice: the first build also pays the CUDA module load of the build kernels ("cold"), the
    # second is the steady-state cost; per-stage device times (CUDA events) of the second.
    def build_canvas():
        if w.op == "knn":
            return None
        if is_dist:
            return sp.Canvas.disks(w.disks["center_xy"], w.disks["r2"], max_dim=a.max_dim or w.max_dim, dense=a.dense)
        return sp.Canvas(w.polys, max_dim=a.max_dim or w.max_dim, dense=a.dense)

    torch.cuda.synchronize()
    t0 = time.perf_counter()
    cv = build_canvas()
    torch.cuda.synchronize()
    build_cold_s = time.perf_counter() - t0
    t0 = time.perf_counter()
    cv2 = build_canvas()
    torch.cuda.synchronize()
    build_s = time.perf_counter() - t0
    if cv is not None:
        cv.close()
    cv = cv2
    info = cv.info() if cv is not None else {}
    build_stages = cv.build_times() if cv is not None else {}
    lc, layers_info = None, None
    if a.layers and w.op == "count" and not is_dist:
        t0 = time.perf_counter()
        lc = sp.LayeredCanvas(w.polys, max_dim=a.max_dim or w.max_dim)
        torch.cuda.synchronize()
        layers_info = {"num_layers": lc.num_layers, "build_s": time.perf_counter() - t0,
                       "plan": "layer index: one canvas and one probe pass per layer (spade_join_count_layered)"}

    # this rank's shard: global indices [rank*n, (rank+1)*n), generated in place on the device
    xy = torch.empty((n, 2), dtype=torch.int32, device=dev)
    gen.points_device(w.points, w.point_seed, rank * n, n, out=xy)
    counts = torch.zeros(P, dtype=torch.int64, device=dev)
    op = w.op
    out_sel = torch.empty(n, dtype=torch.int64, device=dev) if op == "select" else None
    out_pairs = (torch.empty(n, dtype=torch.int64, device=dev), torch.empty(n, dtype=torch.int32, device=dev)) \
        if op == "pairs" else None
    torch.cuda.synchronize()
    n_results = [0]

    def step(ev_k0=None, ev_k1=None):
        if op == "count":
            counts.zero_()
        if ev_k0 is not None:
            ev_k0.record(stream)
        if op == "count":
            if lc is not None:
                sp.join_count_layered(lc, xy, counts)
            else:
                sp.join_count(cv, xy, counts)
        elif op == "knn":
            n_results[0] = sp.knn(xy, w.query, w.k, point_id_base=rank * n)[0].numel()
        elif op == "select":
            n_results[0] = sp.select(cv, xy, point_id_base=rank * n, out=out_sel).numel()
        else:
            n_results[0] = sp.join_pairs(cv, xy, point_id_base=rank * n, out=out_pairs)[0].numel()
        if ev_k1 is not None:
            ev_k1.record(stream)
        if ws > 1 and op == "count":
            dist.all_reduce(counts)

    for _ in range(max(3, a.warmup)):
        step()
    torch.cuda.synchronize()
    sampler = ClockSampler(local)
    if not a.profile:
        sampler.start()
    kev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    l0 = sp.launch_count()
    e0.record(stream)
    for k in range(a.steps):
        step(*kev[k])
    e1.record(stream)
    torch.cuda.synchronize()
    l1 = sp.launch_count()
    if ws > 1:
        dist.barrier()
    clocks = sampler.stop() if not a.profile else None
    t_ms = e0.elapsed_time(e1)
    kern_ms = [s.elapsed_time(t) for s, t in kev]
    # per-stage breakdown of one more (untimed) step: CUDA events between the library's stages
    stage_ms = None
    if op in ("count", "select", "pairs"):
        sp.set_option("stage_events", 1)
        step()
        torch.cuda.synchronize()
        stage_ms = sp.last_call_stages()
        sp.set_option("stage_events", 0)
    t_max = t_ms
    if ws > 1:
        tt = torch.tensor([t_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_max = tt.item()
    total_pts = n * ws
    value = total_pts * a.steps / (t_max / 1e3)
    # correctness guard: tilings cover the whole domain, every point is counted exactly once
    if op == "count" and is_dist:
        check = {"pairs_counted": int(counts.sum().item())}
    elif op == "count":
        check = {"sum_counts_equals_points": int(counts.sum().item()) == total_pts}
    elif op == "pairs" and is_dist:
        check = {"pairs": n_results[0], "pairs_per_point": n_results[0] / n}
    elif op == "pairs":
        check = {"one_pair_per_point": n_results[0] == n}
    elif op == "knn":
        check = {"k_returned": n_results[0], "k": w.k, "note": "single-GPU kNN per rank (N>1: per-shard)"}
    else:
        check = {"selected": n_results[0], "selectivity": n_results[0] / n}
    if lc is not None:
        # the layered plan's counts (the last step's) against the owner-set canvas on the same shard
        ref = torch.zeros(P, dtype=torch.int64, device=dev)
        sp.join_count(cv, xy, ref)
        if ws > 1:
            dist.all_reduce(ref)
        check["layers_equal_owner_sets"] = bool(torch.equal(ref, counts))

    kavg = statistics.mean(kern_ms)
    peak, peak_src = measured_peak()
    # a same-run streaming-READ reference over the same 8 B/point buffer (the copy peak of
    # MEASURED_PEAKS.json counts read + write bytes; a read-only stream can exceed it): the best
    # of 5 float32 sums over the points buffer (a lower bound of the read peak; the round-1
    # microbenchmark tools/microbench/probe_mb.cu read 7,100 GB/s on this pool)
    read_gbs = None
    if op in ("count", "select", "pairs", "knn"):
        rv = xy.view(torch.float32)
        best = None
        for _ in range(5):
            r0, r1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            r0.record(stream)
            rv.sum()
            r1.record(stream)
            torch.cuda.synchronize()
            t = r0.elapsed_time(r1)
            best = t if best is None else min(best, t)
        read_gbs = rv.numel() * 4 / (best / 1e3) / 1e9
    # algorithmic bytes per launch: the int2 stream, plus the results written (select: 8 B id per
    # selected point; pairs: 8 B id + 4 B polygon id per pair); counts are 8*P bytes, negligible
    # kNN: two passes over the points (circle aggregation, distance selection)
    out_bytes = {"count": 0, "select": 8 * n_results[0], "pairs": 12 * n_results[0], "knn": n * 8}[op]
    alg_bytes = n * 8 + out_bytes
    achieved = alg_bytes / (kavg / 1e3) / 1e9
    traffic, traffic_src = ncu_traffic(w.name) if lc is None else (None, None)

    line = None
    if rank == 0:
        line = {
            "metric": METRICS[("dist_" + op) if is_dist and op != "knn" else op], "value": value, "unit": "points/s", "n_gpus": ws, "steps": a.steps,
            "warmup": max(3, a.warmup), "ms_per_step": t_max / a.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {
                "workload": w.name, "desc": w.desc, "points_per_gpu": n,
                **({"disks": P} if is_dist and op != "knn" else {"k": w.k, "query": list(w.query)} if op == "knn"
                   else {"polygons": P, "vertices": int(len(w.polys["ring_xy"]))}),
                "parallelism": f"dp{ws} (points sharded, canvas replicated)",
                "l2": "inputs (8 B/point, >= 8 GB per GPU) exceed the 126 MB L2; no flush needed",
                **({"layers": layers_info} if layers_info else {}),
                "canvas": info, "canvas_build_s": build_s, "canvas_build_cold_s": build_cold_s,
                "canvas_build_stage_ms": build_stages,
                **({"options": a.opt} if a.opt else {}),
            },
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic,
                         "frac_of_read_peak": achieved / max(7100.0, read_gbs or 0.0),
                         "read_peak": {"same_run_torch_sum_gbs": read_gbs, "microbenchmark_gbs": 7100.0,
                                       "note": "frac_of_read_peak divides by the larger of the two"},
                         "kernel": {"knn": "k_knn_hist + k_knn_select + top-k sort (spade_knn; includes its host syncs)",
                                    "count": "k_probe<COUNT> (spade_join_count)",
                                    "select": "k_probe<SELECT> (spade_select; includes its n_out readback)",
                                    "pairs": "k_probe<PAIRS> (spade_join_pairs; includes its n_out readback)"}[op],
                         "kernel_ms": kavg, "algorithmic_bytes_per_launch": alg_bytes, "peak_source": peak_src,
                         "traffic_source": traffic_src},
            "gpu_launches": int(l1 - l0),
            "stages_ms": stage_ms,
            "check": check,
        }
        if clocks:
            line["clocks"] = clocks

    # end-to-end through the public API from pinned host memory (H2D + D2H inside the timing):
    # every rank streams its own shard from host memory, then the counts all_reduce; max over ranks
    if not a.no_e2e and not a.profile and op == "count":
        host = torch.empty((n, 2), dtype=torch.int32, pin_memory=True)
        host.copy_(xy)
        del xy
        torch.cuda.empty_cache()
        hc = np.zeros(P, dtype=np.int64)
        sp.join_count_host(cv, host, hc)   # warm-up
        times = []
        for _ in range(a.e2e_steps):
            hc[:] = 0
            if ws > 1:
                dist.barrier()
            torch.cuda.synchronize()
            s0 = time.perf_counter()
            sp.join_count_host(cv, host, hc)
            if ws > 1:
                ct = torch.from_numpy(hc).to(dev)
                dist.all_reduce(ct)
                hc[:] = ct.cpu().numpy()
            dt = time.perf_counter() - s0
            if ws > 1:
                tt = torch.tensor([dt], dtype=torch.float64, device=dev)
                dist.all_reduce(tt, op=dist.ReduceOp.MAX)
                dt = tt.item()
            times.append(dt)
        if rank == 0:
            line["e2e"] = {"value": total_pts / statistics.median(times), "unit": "points/s",
                           "h2d_bytes_per_step": n * 8, "d2h_bytes_per_step": P * 8,
                           "api": "spade_join_count_host (pinned host buffer per rank) + all_reduce",
                           "steps": a.e2e_steps, "ok": int(hc.sum()) == total_pts,
                           "timing": "host wall clock around the synchronous API call, max over ranks"}
    elif not a.no_e2e and not a.profile and op in ("pairs", "select"):
        # SELECT / PAIRS from pinned host memory into pinned host result arrays
        # (spade_select_host / spade_join_pairs_host: chunked H2D, probe and result D2H overlapped)
        host = torch.empty((n, 2), dtype=torch.int32, pin_memory=True)
        host.copy_(xy)
        del xy
        torch.cuda.empty_cache()
        cap = n
        hpt = torch.empty(cap, dtype=torch.int64, pin_memory=True)
        hpl = torch.empty(cap, dtype=torch.int32, pin_memory=True) if op == "pairs" else None

        def e2e_call():
            if op == "pairs":
                r = sp.join_pairs_host(cv, host, rank * n, capacity=cap, out=(hpt, hpl))
                return len(r[0])
            return len(sp.select_host(cv, host, rank * n, capacity=cap, out=hpt))

        m = e2e_call()   # warm-up
        times = []
        for _ in range(a.e2e_steps):
            if ws > 1:
                dist.barrier()
            torch.cuda.synchronize()
            s0 = time.perf_counter()
            m = e2e_call()
            dt = time.perf_counter() - s0
            if ws > 1:
                tt = torch.tensor([dt], dtype=torch.float64, device=dev)
                dist.all_reduce(tt, op=dist.ReduceOp.MAX)
                dt = tt.item()
            times.append(dt)
        if rank == 0:
            per = 12 if op == "pairs" else 8
            line["e2e"] = {"value": total_pts / statistics.median(times), "unit": "points/s",
                           "h2d_bytes_per_step": n * 8, "d2h_bytes_per_step": m * per,
                           "api": f"spade_{'join_pairs' if op == 'pairs' else 'select'}_host (pinned host "
                                  "points -> pinned host results, per rank)",
                           "steps": a.e2e_steps, "results": m, "ok": m == n_results[0],
                           "timing": "host wall clock around the synchronous API call, max over ranks"}
    elif rank == 0 and not a.profile:
        line["e2e"] = None
    if rank == 0 and not a.no_cpu_baseline and not a.profile and ws == 1:
        cb = cpu_oracle_rate(w, a.cpu_seconds)
        cb.pop("seconds", None)
        cb.pop("sum_counts", None)
        idx, ocounts, rate = cb.pop("idx"), cb.pop("counts", None), cb.pop("rate")
        line["cpu_baseline"] = cb
        if not is_dist:
            line["cpu_rtree_baseline"] = cpu_rtree_rate(w, a.cpu_seconds / 2)
        if not a.no_parity:
            line["parity"] = parity_check(w, cv, sp, idx, ocounts, rate)
    elif rank == 0 and not a.profile and not a.no_parity:
        # N > 1 (or no CPU baseline): the parity check alone, on a small strided sample of the
        # global stream (all ranks' points), rank 0
        import numpy as np
        m = 2000 if w.name.startswith("c5") else 20000
        stride = max(1, (n * ws) // m)
        line["parity"] = parity_check(w, cv, sp, np.arange(m, dtype=np.int64) * stride + 1, None, None)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
