"""Build libspade.so (the CUDA path + C ABI) in-tree for sm_100a with nvcc."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libspade.so")
SOURCES = ["spade_api.cu", "canvas_build.cu", "probe.cu", "knn.cu", "polygon_join.cu", "layers.cu"]
NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
              "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC,-fvisibility=hidden", "-Xptxas", "-v"]


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    srcs = [os.path.join(CSRC, s) for s in SOURCES]
    deps = srcs + [os.path.abspath(__file__), os.path.join(CSRC, "spade_internal.cuh"), os.path.join(ROOT, "include", "spade.h")]
    if not force and not _stale(LIB, deps):
        return LIB
    # Each translation unit is its own device module (no device link across them): CUDA's lazy
    # loading then loads only the module of the kernels a call uses -- a first canvas build loads
    # the builder's ~1 MB module, not the probe's ~16 MB (C5 cold build 2.0 s -> see DESIGN.md).
    # probe.cu keeps separate compilation (-dc + its own device link: its register allocation
    # was tuned that way).
    def compile_one(s):
        o = os.path.join(CSRC, os.path.basename(s).replace(".cu", ".o"))
        rdc = os.path.basename(s) == "probe.cu"
        cmd = ["nvcc", *NVCC_FLAGS, "-I", os.path.join(ROOT, "include"), "-dc" if rdc else "-c", "-o", o, s]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {s}:\n{r.stdout}\n{r.stderr}")
        if verbose:
            print(r.stderr)
        out = [o]
        if rdc:
            dl = o.replace(".o", "_dlink.o")
            cmd = ["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-Xcompiler", "-fPIC", "-dlink", "-o", dl, o]
            r = subprocess.run(cmd, capture_output=True, text=True)
            if r.returncode != 0:
                raise RuntimeError(f"device link failed for {s}:\n{r.stdout}\n{r.stderr}")
            out.append(dl)
        return out

    # the translation units compile in parallel (probe.cu, the longest, first)
    from concurrent.futures import ThreadPoolExecutor
    order = sorted(srcs, key=lambda s: os.path.basename(s) != "probe.cu")
    with ThreadPoolExecutor(max_workers=min(len(order), os.cpu_count() or 1)) as ex:
        done = dict(zip(order, ex.map(compile_one, order)))
    objs = [o for s in srcs for o in done[s]]
    cmd = ["g++", "-shared", "-fPIC", "-o", LIB, *objs, "-L/usr/local/cuda/lib64", "-lcudadevrt", "-lcudart_static", "-lrt", "-lpthread", "-ldl"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
