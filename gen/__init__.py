"""Seeded synthetic inputs shared by the oracle side and the CUDA side (input data only).

Points: counter-based generator in ``spade_gen.h`` (``pt(params, seed, global_index)``), driven
on the device by ``libspade_gen.so:sg_points_device`` and on the host by ``sg_points_host`` /
``sg_points_at`` — bit-identical.  Polygons: ``gen.polygons`` (numpy, host).  Workload recipes
for BASELINE.json's five configs: ``gen.configs``.  Nothing here computes a join.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libspade_gen.so")
_lib = None

SG_MAX_CLUSTERS = 64
KIND_UNIFORM, KIND_TAXI = 0, 1
DOMAIN = 1 << 24


class SgParams(ctypes.Structure):
    _fields_ = [
        ("kind", ctypes.c_int32), ("ncl", ctypes.c_int32),
        ("x0", ctypes.c_int32), ("y0", ctypes.c_int32), ("w", ctypes.c_int32), ("h", ctypes.c_int32),
        ("bg_thresh", ctypes.c_uint32),
        ("cum", ctypes.c_uint32 * SG_MAX_CLUSTERS),
        ("cx", ctypes.c_int32 * SG_MAX_CLUSTERS), ("cy", ctypes.c_int32 * SG_MAX_CLUSTERS),
        ("sx", ctypes.c_int32 * SG_MAX_CLUSTERS), ("sy", ctypes.c_int32 * SG_MAX_CLUSTERS),
        ("shear", ctypes.c_int32 * SG_MAX_CLUSTERS),
    ]


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "gen_lib.cu")
    hdr = os.path.join(_HERE, "spade_gen.h")
    newest = max(os.path.getmtime(src), os.path.getmtime(hdr))
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < newest:
        subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo",
                               "-shared", "-Xcompiler", "-fPIC", "-o", _LIB_PATH, src])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        P = ctypes.c_void_p
        lib.sg_points_device.argtypes = [P, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int64, P, P]
        lib.sg_points_device.restype = ctypes.c_int
        lib.sg_points_host.argtypes = [P, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int64, P]
        lib.sg_points_host.restype = None
        lib.sg_points_at.argtypes = [P, ctypes.c_uint64, P, ctypes.c_int64, P]
        lib.sg_points_at.restype = None
        lib.sg_params_size.restype = ctypes.c_int
        assert lib.sg_params_size() == ctypes.sizeof(SgParams), "sg_params layout mismatch"
        _lib = lib
    return _lib


def uniform_params(x0: int, y0: int, w: int, h: int) -> SgParams:
    p = SgParams()
    p.kind, p.x0, p.y0, p.w, p.h = KIND_UNIFORM, x0, y0, w, h
    return p


def taxi_params(seed: int, domain: int = DOMAIN, ncl: int = 64, zipf: float = 1.1,
                bg_frac: float = 0.10) -> SgParams:
    """"Taxi-like" clustered points (Table 1, Taxi P:279): Zipf(1.1) cluster weights,
    centres uniform in the central 60% of the domain, spreads log-uniform in [2^14, 2^19] with
    random aspect, a quarter of the clusters sheared into streaks, 10% uniform background."""
    rng = np.random.default_rng(seed)
    p = SgParams()
    p.kind, p.ncl, p.x0, p.y0, p.w, p.h = KIND_TAXI, ncl, 0, 0, domain, domain
    p.bg_thresh = int(bg_frac * 2**32)
    w = 1.0 / np.arange(1, ncl + 1, dtype=np.float64) ** zipf
    cum = np.floor(np.cumsum(w) / w.sum() * 2**32).astype(np.uint64)
    cum = np.minimum(cum, 2**32 - 1)
    cum[-1] = 2**32 - 1
    lo, hi = int(0.2 * domain), int(0.8 * domain)
    for k in range(ncl):
        p.cum[k] = int(cum[k])
        p.cx[k] = int(rng.integers(lo, hi))
        p.cy[k] = int(rng.integers(lo, hi))
        s = 2.0 ** rng.uniform(14, 19)
        aspect = 2.0 ** rng.uniform(-1, 1)
        p.sx[k] = int(s * aspect ** 0.5)
        p.sy[k] = int(s / aspect ** 0.5)
        p.shear[k] = int(rng.integers(-512, 513)) if rng.random() < 0.25 else 0
    return p


def points_host(params: SgParams, seed: int, start: int, n: int) -> np.ndarray:
    """Points with global indices [start, start+n) as an (n, 2) int32 array."""
    lib = _load()
    out = np.empty((n, 2), dtype=np.int32)
    if n:
        lib.sg_points_host(ctypes.byref(params), seed, start, n, out.ctypes.data_as(ctypes.c_void_p))
    return out


def points_at(params: SgParams, seed: int, indices) -> np.ndarray:
    """Points at arbitrary global indices as an (m, 2) int32 array."""
    lib = _load()
    idx = np.ascontiguousarray(indices, dtype=np.int64)
    out = np.empty((len(idx), 2), dtype=np.int32)
    if len(idx):
        lib.sg_points_at(ctypes.byref(params), seed, idx.ctypes.data_as(ctypes.c_void_p), len(idx),
                         out.ctypes.data_as(ctypes.c_void_p))
    return out


def points_device(params: SgParams, seed: int, start: int, n: int, out=None, stream=None):
    """Points [start, start+n) generated in place into a CUDA int32 tensor of shape (n, 2)."""
    import torch
    lib = _load()
    if out is None:
        out = torch.empty((n, 2), dtype=torch.int32, device="cuda")
    assert out.is_cuda and out.dtype == torch.int32 and out.is_contiguous() and out.numel() >= 2 * n
    s = stream if stream is not None else torch.cuda.current_stream()
    rc = lib.sg_points_device(ctypes.byref(params), seed, start, n, ctypes.c_void_p(out.data_ptr()),
                              ctypes.c_void_p(s.cuda_stream))
    if rc != 0:
        raise RuntimeError("sg_points_device launch failed")
    return out
