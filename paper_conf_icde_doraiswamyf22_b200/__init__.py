"""paper_conf_icde_doraiswamyf22_b200 — B200-native SPADE point-in-polygon join (thin binding).

Argument marshalling only: every step of the path runs in libspade.so (CUDA kernels for sm_100a
behind the C ABI of include/spade.h).  PyTorch supplies device memory and streams.  There is no
CPU fallback: if the extension cannot be loaded, or no CUDA device is present, calls raise.

    canvas = Canvas(polys)                       # spade_build_canvas   (Sec. 4.2-4.3)
    counts = join_count(canvas, xy)              # spade_join_count     (aggregation)
    ids    = select(canvas, xy)                  # spade_select         (selection)
    pt, pl = join_pairs(canvas, xy)              # spade_join_pairs     (join)
    counts = join_count_host(canvas, xy_numpy)   # spade_join_count_host (host-resident points)
    dcv    = Canvas.disks(centers, r2)           # spade_build_disk_canvas (distance canvas)
    ids, d2 = knn(xy, (qx, qy), k)               # spade_knn              (kNN selection)

`polys` is a dict with ``ring_xy`` (V,2) int32, ``ring_off`` (R+1) int64, ``poly_ring_off``
(P+1) int64 (numpy arrays or torch tensors), the layout spade_build_canvas takes.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libspade.so")
_lib = None

SPADE_OK, SPADE_ERR_INVALID_ARG, SPADE_ERR_COORD_RANGE = 0, -1, -2
SPADE_ERR_CAPACITY, SPADE_ERR_CUDA, SPADE_ERR_OOM, SPADE_ERR_INTERNAL = -3, -4, -5, -6


class SpadeError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"spade error {code}: {msg}")
        self.code = code


class CapacityError(SpadeError):
    def __init__(self, code, msg, needed):
        super().__init__(code, msg)
        self.needed = needed


class CanvasParams(ctypes.Structure):
    _fields_ = [("log2_pixel", ctypes.c_int32), ("max_dim", ctypes.c_int32), ("flags", ctypes.c_int32)]


SPADE_CANVAS_DENSE = 1


def load(path: str | None = None):
    """Load libspade.so (build it first with __graft_entry__.build()); raises if missing."""
    global _lib
    if _lib is not None:
        return _lib
    p = path or LIB_PATH
    if not os.path.exists(p):
        raise ImportError(f"libspade.so not built ({p}); run `python -c 'import __graft_entry__ as g; g.build()'`")
    lib = ctypes.CDLL(p)
    P, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    lib.spade_build_canvas.argtypes = [P, P, P, i32, ctypes.POINTER(CanvasParams), P, ctypes.POINTER(P)]
    lib.spade_build_canvas.restype = ctypes.c_int
    lib.spade_build_disk_canvas.argtypes = [P, P, i32, ctypes.POINTER(CanvasParams), P, ctypes.POINTER(P)]
    lib.spade_build_disk_canvas.restype = ctypes.c_int
    lib.spade_canvas_free.argtypes = [P]
    lib.spade_canvas_free.restype = None
    lib.spade_canvas_info.argtypes = [P] + [ctypes.POINTER(i32)] * 6 + [ctypes.POINTER(i64)] * 2 + [ctypes.POINTER(ctypes.c_double)]
    lib.spade_canvas_info.restype = ctypes.c_int
    lib.spade_join_polygons.argtypes = [P, P, P, i32, P, P, P, i32, ctypes.POINTER(CanvasParams), P, P, i64,
                                         ctypes.POINTER(i64), P]
    lib.spade_join_polygons.restype = ctypes.c_int
    lib.spade_canvas_build_times.argtypes = [P, ctypes.POINTER(ctypes.c_float), i32]
    lib.spade_canvas_build_times.restype = ctypes.c_int
    lib.spade_canvas_build_stage_name.argtypes = [i32]
    lib.spade_canvas_build_stage_name.restype = ctypes.c_char_p
    lib.spade_canvas_checksum.argtypes = [P, ctypes.POINTER(ctypes.c_uint64), P]
    lib.spade_canvas_checksum.restype = ctypes.c_int
    lib.spade_join_count.argtypes = [P, P, i64, P, P]
    lib.spade_join_count.restype = ctypes.c_int
    lib.spade_select.argtypes = [P, P, i64, i64, P, i64, ctypes.POINTER(i64), P]
    lib.spade_select.restype = ctypes.c_int
    lib.spade_join_pairs.argtypes = [P, P, i64, i64, P, P, i64, ctypes.POINTER(i64), P]
    lib.spade_join_pairs.restype = ctypes.c_int
    lib.spade_join_count_host.argtypes = [P, P, i64, P, P]
    lib.spade_join_count_host.restype = ctypes.c_int
    lib.spade_select_host.argtypes = [P, P, i64, i64, P, i64, ctypes.POINTER(i64), P]
    lib.spade_select_host.restype = ctypes.c_int
    lib.spade_join_pairs_host.argtypes = [P, P, i64, i64, P, P, i64, ctypes.POINTER(i64), P]
    lib.spade_join_pairs_host.restype = ctypes.c_int
    lib.spade_knn_histogram.argtypes = [P, i64, i32, i32, P, P]
    lib.spade_knn_histogram.restype = ctypes.c_int
    lib.spade_knn_radius.argtypes = [P, i64, ctypes.POINTER(i64), ctypes.POINTER(i64)]
    lib.spade_knn_radius.restype = ctypes.c_int
    lib.spade_knn_select.argtypes = [P, i64, i64, i32, i32, i64, P, P, i64, ctypes.POINTER(i64), P]
    lib.spade_knn_select.restype = ctypes.c_int
    lib.spade_knn_topk.argtypes = [P, P, i64, i64, P, P, P]
    lib.spade_knn_topk.restype = ctypes.c_int
    lib.spade_knn.argtypes = [P, i64, i64, i32, i32, i64, P, P, ctypes.POINTER(i64), P]
    lib.spade_knn.restype = ctypes.c_int
    lib.spade_layer_assign.argtypes = [P, P, i64, i32, P, ctypes.POINTER(i32)]
    lib.spade_layer_assign.restype = ctypes.c_int
    lib.spade_build_layered.argtypes = [P, P, P, i32, ctypes.POINTER(CanvasParams), P, ctypes.POINTER(P)]
    lib.spade_build_layered.restype = ctypes.c_int
    lib.spade_join_count_layered.argtypes = [P, P, i64, P, P]
    lib.spade_join_count_layered.restype = ctypes.c_int
    lib.spade_layered_info.argtypes = [P, ctypes.POINTER(i32), P]
    lib.spade_layered_info.restype = ctypes.c_int
    lib.spade_layered_free.argtypes = [P]
    lib.spade_layered_free.restype = None
    lib.spade_set_option.argtypes = [ctypes.c_char_p, i64]
    lib.spade_set_option.restype = ctypes.c_int
    lib.spade_last_call_stages.argtypes = [ctypes.POINTER(ctypes.c_float), i32]
    lib.spade_last_call_stages.restype = ctypes.c_int
    lib.spade_launch_count.argtypes = []
    lib.spade_launch_count.restype = i64
    lib.spade_status_string.argtypes = [ctypes.c_int]
    lib.spade_status_string.restype = ctypes.c_char_p
    lib.spade_last_error.argtypes = []
    lib.spade_last_error.restype = ctypes.c_char_p
    _lib = lib
    return lib


EXPORTED_SYMBOLS = ["spade_build_canvas", "spade_build_disk_canvas", "spade_canvas_free", "spade_canvas_info",
                    "spade_canvas_checksum", "spade_canvas_build_times", "spade_canvas_build_stage_name", "spade_join_polygons", "spade_join_count",
                    "spade_select", "spade_join_pairs", "spade_join_count_host", "spade_select_host", "spade_join_pairs_host", "spade_knn_histogram",
                    "spade_knn_radius", "spade_knn_select", "spade_knn_topk", "spade_knn", "spade_set_option", "spade_launch_count", "spade_last_call_stages",
                    "spade_status_string", "spade_last_error", "spade_layer_assign", "spade_build_layered",
                    "spade_join_count_layered", "spade_layered_info", "spade_layered_free"]


def _check(rc: int, what: str):
    if rc != SPADE_OK:
        lib = load()
        raise SpadeError(rc, f"{what}: {lib.spade_last_error().decode()}")


def _torch():
    import torch
    if not torch.cuda.is_available():
        raise RuntimeError("paper_conf_icde_doraiswamyf22_b200 needs a CUDA device (no CPU fallback)")
    return torch


def _stream(stream):
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _dev(a, dtype, shape_last=None):
    """numpy array / torch tensor -> contiguous CUDA tensor of dtype."""
    torch = _torch()
    t = torch.as_tensor(a) if not isinstance(a, torch.Tensor) else a
    t = t.to(device="cuda", dtype=dtype).contiguous()
    if shape_last is not None:
        t = t.reshape(-1, shape_last)
    return t


def _dev_out(t, dtype, n: int, name: str, device=None):
    """A caller-supplied DEVICE output buffer: must be a contiguous CUDA tensor of `dtype` with
    at least n elements (on `device` if given); the C side writes through its raw pointer."""
    torch = _torch()
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor")
    if t.dtype != dtype:
        raise ValueError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    if t.numel() < n:
        raise ValueError(f"{name} holds {t.numel()} elements, needs >= {n}")
    if device is not None and t.device != device:
        raise ValueError(f"{name} is on {t.device}, the canvas on {device}")
    return t


def _host_buf(a, dtype, n: int, name: str):
    """A caller-supplied HOST buffer (numpy array or CPU tensor): dtype, C-contiguous, writeable,
    >= n elements; returns its address."""
    if hasattr(a, "data_ptr"):
        torch = _torch()
        if a.is_cuda:
            raise ValueError(f"{name} must be a host (CPU) tensor")
        if a.dtype != {np.int64: torch.int64, np.int32: torch.int32}[dtype]:
            raise ValueError(f"{name} must be {np.dtype(dtype).name}, got {a.dtype}")
        if not a.is_contiguous():
            raise ValueError(f"{name} must be contiguous")
        if a.numel() < n:
            raise ValueError(f"{name} holds {a.numel()} elements, needs >= {n}")
        return a.data_ptr()
    if not isinstance(a, np.ndarray):
        raise ValueError(f"{name} must be a numpy array or a CPU tensor")
    if a.dtype != np.dtype(dtype):
        raise ValueError(f"{name} must be {np.dtype(dtype).name}, got {a.dtype}")
    if not a.flags.c_contiguous or not a.flags.writeable:
        raise ValueError(f"{name} must be C-contiguous and writeable")
    if a.size < n:
        raise ValueError(f"{name} holds {a.size} elements, needs >= {n}")
    return a.ctypes.data


def set_option(name: str, value: int) -> None:
    """Probe-path tuning option (include/spade.h spade_set_option); results never depend on it."""
    _check(load().spade_set_option(name.encode(), int(value)), f"set_option({name})")


PROBE_STAGES = ["probe", "deferred exact tests", "output compaction", "counter expansion"]


def last_call_stages() -> dict:
    """Per-stage device ms of this thread's last COUNT / SELECT / PAIRS call (needs
    set_option("stage_events", 1) before the call; spade_last_call_stages)."""
    ms = (ctypes.c_float * 4)()
    load().spade_last_call_stages(ms, 4)
    return {k: float(v) for k, v in zip(PROBE_STAGES, ms)}


def launch_count() -> int:
    return int(load().spade_launch_count())


class Canvas:
    """Discrete canvas + boundary index of a polygon set (owns device memory).
    ``Canvas.disks(...)`` builds a distance canvas (one closed disk per constraint) instead."""

    def __init__(self, polys, log2_pixel: int = -1, max_dim: int = 4096, dense: bool = False, stream=None):
        torch = _torch()
        lib = load()
        self.device = torch.device("cuda", torch.cuda.current_device())
        if polys is None:                    # filled in by Canvas.disks
            self._h, self._lib, self.num_polys = None, lib, 0
            return
        ring_xy = _dev(polys["ring_xy"], torch.int32, 2)
        ring_off = _dev(polys["ring_off"], torch.int64)
        poly_ring_off = _dev(polys["poly_ring_off"], torch.int64)
        self.num_polys = int(poly_ring_off.numel()) - 1
        prm = CanvasParams(log2_pixel, max_dim, SPADE_CANVAS_DENSE if dense else 0)
        h = ctypes.c_void_p()
        rc = lib.spade_build_canvas(ctypes.c_void_p(ring_xy.data_ptr()), ctypes.c_void_p(ring_off.data_ptr()),
                                    ctypes.c_void_p(poly_ring_off.data_ptr()), self.num_polys, ctypes.byref(prm),
                                    _stream(stream), ctypes.byref(h))
        _check(rc, "spade_build_canvas")
        self._h = h
        self._lib = lib

    @classmethod
    def disks(cls, center_xy, r2, log2_pixel: int = -1, max_dim: int = 4096, dense: bool = False, stream=None):
        """Distance canvas (spade_build_disk_canvas): disk d = {p : |p - center_d|^2 <= r2[d]}.
        ``r2`` may be a scalar (type 1 distance join, one radius) or one int64 per disk (type 2)."""
        torch = _torch()
        cxy = _dev(center_xy, torch.int32, 2)
        D = int(cxy.shape[0])
        r2t = torch.as_tensor(r2, dtype=torch.int64)
        if r2t.numel() == 1 and D != 1:
            r2t = r2t.reshape(1).expand(D)
        r2t = r2t.to("cuda").contiguous()
        if r2t.numel() != D:
            raise ValueError("r2 must be a scalar or have one entry per disk")
        self = cls(None)
        prm = CanvasParams(log2_pixel, max_dim, SPADE_CANVAS_DENSE if dense else 0)
        h = ctypes.c_void_p()
        rc = self._lib.spade_build_disk_canvas(ctypes.c_void_p(cxy.data_ptr()), ctypes.c_void_p(r2t.data_ptr()), D,
                                               ctypes.byref(prm), _stream(stream), ctypes.byref(h))
        _check(rc, "spade_build_disk_canvas")
        self._h = h
        self.num_polys = D
        return self

    @property
    def handle(self):
        return self._h

    def info(self) -> dict:
        i32 = [ctypes.c_int32() for _ in range(6)]
        i64 = [ctypes.c_int64() for _ in range(2)]
        d = ctypes.c_double()
        _check(self._lib.spade_canvas_info(self._h, *[ctypes.byref(x) for x in i32],
                                           *[ctypes.byref(x) for x in i64], ctypes.byref(d)), "spade_canvas_info")
        W, H, s, Wc, Hc, b = (x.value for x in i32)
        return {"W": W, "H": H, "log2_pixel": s, "Wc": Wc, "Hc": Hc, "log2_tile": b,
                "num_records": i64[0].value, "num_run_edges": i64[1].value, "mixed_tile_frac": d.value}

    def build_times(self) -> dict:
        """Device time (ms) of each build stage (spade_canvas_build_times; CUDA events)."""
        ms = (ctypes.c_float * 8)()
        n = self._lib.spade_canvas_build_times(self._h, ms, 8)
        if n < 0:
            _check(n, "spade_canvas_build_times")
        return {self._lib.spade_canvas_build_stage_name(i).decode(): float(ms[i]) for i in range(n)}

    def close(self):
        if getattr(self, "_h", None):
            self._lib.spade_canvas_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class LayeredCanvas:
    """The paper's layer index (spade_build_layered): the polygons split
    into layers of mutually non-intersecting polygons (greedy colouring of the closed-intersection
    self-join), one canvas and one probe pass per layer.  The alternative to the owner sets of a
    single Canvas, kept for comparison; polygons must be valid (as for join_polygons)."""

    def __init__(self, polys, log2_pixel: int = -1, max_dim: int = 4096, stream=None):
        torch = _torch()
        lib = load()
        self.device = torch.device("cuda", torch.cuda.current_device())
        ring_xy = _dev(polys["ring_xy"], torch.int32, 2)
        ring_off = _dev(polys["ring_off"], torch.int64)
        poly_ring_off = _dev(polys["poly_ring_off"], torch.int64)
        self.num_polys = int(poly_ring_off.numel()) - 1
        prm = CanvasParams(log2_pixel, max_dim, 0)
        h = ctypes.c_void_p()
        rc = lib.spade_build_layered(ctypes.c_void_p(ring_xy.data_ptr()), ctypes.c_void_p(ring_off.data_ptr()),
                                     ctypes.c_void_p(poly_ring_off.data_ptr()), self.num_polys, ctypes.byref(prm),
                                     _stream(stream), ctypes.byref(h))
        _check(rc, "spade_build_layered")
        self._h, self._lib = h, lib

    @property
    def handle(self):
        return self._h

    @property
    def num_layers(self) -> int:
        L = ctypes.c_int32()
        _check(self._lib.spade_layered_info(self._h, ctypes.byref(L), None), "spade_layered_info")
        return L.value

    def layer_of(self):
        """numpy int32[P]: the layer of every polygon."""
        import numpy as np
        out = np.empty(self.num_polys, dtype=np.int32)
        L = ctypes.c_int32()
        _check(self._lib.spade_layered_info(self._h, ctypes.byref(L), out.ctypes.data_as(ctypes.c_void_p)),
               "spade_layered_info")
        return out

    def close(self):
        if getattr(self, "_h", None):
            self._lib.spade_layered_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def join_count_layered(layered: LayeredCanvas, xy, counts=None, stream=None):
    """Per-polygon COUNT over a layered canvas (spade_join_count_layered: one pass per layer);
    accumulates into `counts` if given."""
    torch = _torch()
    xy, n = _points(xy, layered.device)
    if counts is None:
        counts = torch.zeros(layered.num_polys, dtype=torch.int64, device=layered.device)
    _dev_out(counts, torch.int64, layered.num_polys, "counts", layered.device)
    rc = load().spade_join_count_layered(layered.handle, ctypes.c_void_p(xy.data_ptr()), n,
                                         ctypes.c_void_p(counts.data_ptr()), _stream(stream))
    _check(rc, "spade_join_count_layered")
    return counts


def layer_assign(pair_a, pair_b, num_polys: int):
    """Greedy layer colouring of a conflict graph (spade_layer_assign, host only): numpy int32
    layer_of[num_polys] and the number of layers."""
    import numpy as np
    a = np.ascontiguousarray(pair_a, dtype=np.int32)
    b = np.ascontiguousarray(pair_b, dtype=np.int32)
    if a.shape != b.shape:
        raise ValueError("layer_assign: pair arrays differ in length")
    out = np.empty(max(num_polys, 0), dtype=np.int32)
    L = ctypes.c_int32()
    rc = load().spade_layer_assign(a.ctypes.data_as(ctypes.c_void_p), b.ctypes.data_as(ctypes.c_void_p), len(a),
                                   num_polys, out.ctypes.data_as(ctypes.c_void_p), ctypes.byref(L))
    _check(rc, "spade_layer_assign")
    return out, L.value


def join_polygons(polys1, polys2, capacity: int | None = None, max_dim: int = 4096, log2_pixel: int = -1,
                  stream=None):
    """Polygon x Polygon join (spade_join_polygons): (a, b) int32 CUDA tensors of every
    polygon a of polys1 and b of polys2 whose closed regions intersect, sorted by (a, b)."""
    torch = _torch()
    d = []
    for polys in (polys1, polys2):
        d.append((_dev(polys["ring_xy"], torch.int32, 2), _dev(polys["ring_off"], torch.int64),
                  _dev(polys["poly_ring_off"], torch.int64)))
    n1, n2 = int(d[0][2].numel()) - 1, int(d[1][2].numel()) - 1
    cap = max(n1 + n2, 1024) if capacity is None else int(capacity)
    prm = CanvasParams(log2_pixel, max_dim, 0)
    for _ in range(2):
        a = torch.empty(max(cap, 1), dtype=torch.int32, device="cuda")
        b = torch.empty(max(cap, 1), dtype=torch.int32, device="cuda")
        n_out = ctypes.c_int64()
        args = [ctypes.c_void_p(t.data_ptr()) for t in d[0]] + [n1] + [ctypes.c_void_p(t.data_ptr()) for t in d[1]] + [n2]
        rc = load().spade_join_polygons(*args, ctypes.byref(prm), ctypes.c_void_p(a.data_ptr()),
                                        ctypes.c_void_p(b.data_ptr()), cap, ctypes.byref(n_out), _stream(stream))
        if rc == SPADE_ERR_CAPACITY:
            cap = n_out.value
            continue
        _check(rc, "spade_join_polygons")
        return a[: n_out.value], b[: n_out.value]
    raise SpadeError(SPADE_ERR_CAPACITY, "join_polygons: capacity retry failed")


def canvas_checksum(canvas: Canvas, stream=None) -> int:
    """64-bit checksum of the canvas arrays (spade_canvas_checksum): equal polygon sets give equal
    checksums on every rank (the replicated-canvas check of distributed.canvas_checksums_agree)."""
    h = ctypes.c_uint64()
    _check(load().spade_canvas_checksum(canvas.handle, ctypes.byref(h), _stream(stream)), "spade_canvas_checksum")
    return int(h.value)


def _points(xy, device=None):
    torch = _torch()
    if not (isinstance(xy, torch.Tensor) and xy.is_cuda and xy.dtype == torch.int32 and xy.is_contiguous()):
        xy = _dev(xy, torch.int32, 2) if device is None else \
            (torch.as_tensor(xy) if not isinstance(xy, torch.Tensor) else xy).to(device=device, dtype=torch.int32).contiguous()
    if device is not None and xy.device != device:
        raise ValueError(f"points are on {xy.device}, the canvas on {device}")
    if xy.numel() % 2:
        raise ValueError("points must be (n, 2) int32 coordinates")
    return xy, xy.numel() // 2


def join_count(canvas: Canvas, xy, counts=None, stream=None):
    """Per-polygon COUNT (int64[P] CUDA tensor); accumulates into `counts` if given."""
    torch = _torch()
    xy, n = _points(xy, canvas.device)
    if counts is None:
        counts = torch.zeros(canvas.num_polys, dtype=torch.int64, device=canvas.device)
    _dev_out(counts, torch.int64, canvas.num_polys, "counts", canvas.device)
    rc = load().spade_join_count(canvas.handle, ctypes.c_void_p(xy.data_ptr()), n,
                                 ctypes.c_void_p(counts.data_ptr()), _stream(stream))
    _check(rc, "spade_join_count")
    return counts


def select(canvas: Canvas, xy, point_id_base: int = 0, capacity: int | None = None, stream=None, out=None):
    """int64 CUDA tensor of the ids of points inside >= 1 polygon (order unspecified).
    capacity=None uses n_max = n (1-pass Map); a too-small capacity retries once with the
    reported size (2-pass Map).  `out` (int64 CUDA, >= capacity) avoids the allocation."""
    torch = _torch()
    xy, n = _points(xy, canvas.device)
    cap = n if capacity is None else capacity
    if out is not None:
        _dev_out(out, torch.int64, 0, "out", canvas.device)
    for attempt in range(2):
        if out is None or attempt > 0 or out.numel() < max(cap, 1):
            out = torch.empty(max(cap, 1), dtype=torch.int64, device=canvas.device)
        _dev_out(out, torch.int64, cap, "out", canvas.device)
        n_out = ctypes.c_int64()
        rc = load().spade_select(canvas.handle, ctypes.c_void_p(xy.data_ptr()), n, point_id_base,
                                 ctypes.c_void_p(out.data_ptr()), cap, ctypes.byref(n_out), _stream(stream))
        if rc == SPADE_ERR_CAPACITY:
            cap = n_out.value
            continue
        _check(rc, "spade_select")
        return out[: n_out.value]
    raise SpadeError(SPADE_ERR_CAPACITY, "select: capacity retry failed")


def join_pairs(canvas: Canvas, xy, point_id_base: int = 0, capacity: int | None = None, stream=None, out=None):
    """(point_ids int64, poly_ids int32) CUDA tensors, order unspecified.  `out` = (pt, pl)
    preallocated CUDA tensors (>= capacity) avoids the allocation."""
    torch = _torch()
    xy, n = _points(xy, canvas.device)
    cap = n if capacity is None else capacity
    if out is not None:
        _dev_out(out[0], torch.int64, 0, "out[0]", canvas.device)
        _dev_out(out[1], torch.int32, 0, "out[1]", canvas.device)
    for attempt in range(2):
        if out is not None and attempt == 0 and out[0].numel() >= max(cap, 1) and out[1].numel() >= max(cap, 1):
            pt, pl = out
        else:
            pt = torch.empty(max(cap, 1), dtype=torch.int64, device=canvas.device)
            pl = torch.empty(max(cap, 1), dtype=torch.int32, device=canvas.device)
        _dev_out(pt, torch.int64, cap, "out[0]", canvas.device)
        _dev_out(pl, torch.int32, cap, "out[1]", canvas.device)
        n_out = ctypes.c_int64()
        rc = load().spade_join_pairs(canvas.handle, ctypes.c_void_p(xy.data_ptr()), n, point_id_base,
                                     ctypes.c_void_p(pt.data_ptr()), ctypes.c_void_p(pl.data_ptr()), cap,
                                     ctypes.byref(n_out), _stream(stream))
        if rc == SPADE_ERR_CAPACITY:
            cap = n_out.value
            continue
        _check(rc, "spade_join_pairs")
        return pt[: n_out.value], pl[: n_out.value]
    raise SpadeError(SPADE_ERR_CAPACITY, "join_pairs: capacity retry failed")


def join_count_host(canvas: Canvas, xy_host, counts_host=None, stream=None) -> np.ndarray:
    """COUNT over HOST-resident points (numpy array or pinned CPU tensor); returns int64 numpy."""
    lib = load()
    keep, ptr, n = _host_points(xy_host)
    if counts_host is None:
        counts_host = np.zeros(canvas.num_polys, dtype=np.int64)
    cptr = _host_buf(counts_host, np.int64, canvas.num_polys, "counts_host")
    rc = lib.spade_join_count_host(canvas.handle, ctypes.c_void_p(ptr), n, ctypes.c_void_p(cptr), _stream(stream))
    _check(rc, "spade_join_count_host")
    return counts_host


def _host_points(xy_host):
    if hasattr(xy_host, "data_ptr"):      # torch CPU tensor (pinned for full bandwidth)
        import torch
        if xy_host.is_cuda or not xy_host.is_contiguous() or xy_host.dtype != torch.int32 or xy_host.numel() % 2:
            raise ValueError("host points must be a contiguous (n, 2) int32 CPU tensor")
        return xy_host, xy_host.data_ptr(), xy_host.numel() // 2
    xy_host = np.ascontiguousarray(xy_host, dtype=np.int32)
    return xy_host, xy_host.ctypes.data, xy_host.size // 2


def _host_out(out, cap, dtype):
    """Caller's host output array (numpy or CPU tensor, pinned for full bandwidth) if it holds
    `cap` elements, else a new numpy array; returns (array, address)."""
    if out is not None:
        size = out.numel() if hasattr(out, "data_ptr") else np.asarray(out).size
        if size >= cap:
            return out, _host_buf(out, dtype, cap, "out")
        _host_buf(out, dtype, 0, "out")            # type errors are reported even when too small
    a = np.empty(max(cap, 1), dtype=dtype)
    return a, a.ctypes.data


def select_host(canvas: Canvas, xy_host, point_id_base: int = 0, capacity: int | None = None, stream=None,
                out=None):
    """SELECT over HOST-resident points (spade_select_host): int64 ids (numpy, or `out`'s type
    when a large enough host array / pinned CPU tensor is given), chunk order.
    capacity=None is n_max = n; a too-small capacity retries with the reported size."""
    _torch()
    keep, ptr, n = _host_points(xy_host)
    cap = n if capacity is None else capacity
    for attempt in range(2):
        out, optr = _host_out(out if attempt == 0 else None, cap, np.int64)
        n_out = ctypes.c_int64()
        rc = load().spade_select_host(canvas.handle, ctypes.c_void_p(ptr), n, point_id_base,
                                      ctypes.c_void_p(optr), cap, ctypes.byref(n_out), _stream(stream))
        if rc == SPADE_ERR_CAPACITY:
            cap = n_out.value
            continue
        _check(rc, "spade_select_host")
        return out[: n_out.value]
    raise SpadeError(SPADE_ERR_CAPACITY, "select_host: capacity retry failed")


def join_pairs_host(canvas: Canvas, xy_host, point_id_base: int = 0, capacity: int | None = None, stream=None,
                    out=None):
    """PAIRS over HOST-resident points (spade_join_pairs_host): (int64 point ids, int32 polygon
    ids) host arrays; `out` = (pt, pl) preallocated host arrays / pinned CPU tensors."""
    _torch()
    keep, ptr, n = _host_points(xy_host)
    cap = n if capacity is None else capacity
    for attempt in range(2):
        pt, ptp = _host_out(out[0] if out is not None and attempt == 0 else None, cap, np.int64)
        pl, plp = _host_out(out[1] if out is not None and attempt == 0 else None, cap, np.int32)
        n_out = ctypes.c_int64()
        rc = load().spade_join_pairs_host(canvas.handle, ctypes.c_void_p(ptr), n, point_id_base,
                                          ctypes.c_void_p(ptp), ctypes.c_void_p(plp), cap,
                                          ctypes.byref(n_out), _stream(stream))
        if rc == SPADE_ERR_CAPACITY:
            cap = n_out.value
            continue
        _check(rc, "spade_join_pairs_host")
        return pt[: n_out.value], pl[: n_out.value]
    raise SpadeError(SPADE_ERR_CAPACITY, "join_pairs_host: capacity retry failed")


# ---- kNN selection (spade_knn*): circles -> aggregation -> distance select -> sort ----
KNN_BINS = 248


def knn_histogram(xy, q, hist=None, stream=None):
    """Step 1: int64[KNN_BINS + 1] CUDA tensor of squared-distance bucket counts (accumulated
    into `hist` if given); the last entry counts points outside [-2^30, 2^30)."""
    torch = _torch()
    xy, n = _points(xy)
    if hist is None:
        hist = torch.zeros(KNN_BINS + 1, dtype=torch.int64, device="cuda")
    _check(load().spade_knn_histogram(ctypes.c_void_p(xy.data_ptr()), n, int(q[0]), int(q[1]),
                                      ctypes.c_void_p(hist.data_ptr()), _stream(stream)), "spade_knn_histogram")
    return hist


def knn_radius(hist_host, k: int):
    """(r2, count): the smallest circle holding >= k points, from a host histogram."""
    h = np.ascontiguousarray(np.asarray(hist_host, dtype=np.int64))
    r2, cnt = ctypes.c_int64(), ctypes.c_int64()
    _check(load().spade_knn_radius(h.ctypes.data_as(ctypes.c_void_p), int(k), ctypes.byref(r2), ctypes.byref(cnt)),
           "spade_knn_radius")
    return r2.value, cnt.value


def knn_select(xy, q, r2: int, point_id_base: int = 0, capacity: int | None = None, stream=None):
    """Step 2: (ids, d2) int64 CUDA tensors of the points with dist2 <= r2 (order unspecified)."""
    torch = _torch()
    xy, n = _points(xy)
    cap = n if capacity is None else capacity
    for _ in range(2):
        ids = torch.empty(max(cap, 1), dtype=torch.int64, device="cuda")
        d2 = torch.empty(max(cap, 1), dtype=torch.int64, device="cuda")
        n_out = ctypes.c_int64()
        rc = load().spade_knn_select(ctypes.c_void_p(xy.data_ptr()), n, point_id_base, int(q[0]), int(q[1]), int(r2),
                                     ctypes.c_void_p(ids.data_ptr()), ctypes.c_void_p(d2.data_ptr()), cap,
                                     ctypes.byref(n_out), _stream(stream))
        if rc == SPADE_ERR_CAPACITY:
            cap = n_out.value
            continue
        _check(rc, "spade_knn_select")
        return ids[: n_out.value], d2[: n_out.value]
    raise SpadeError(SPADE_ERR_CAPACITY, "knn_select: capacity retry failed")


def knn_topk(ids, d2, k: int, stream=None):
    """Step 3: the first min(k, m) candidates in (d2, id) order, as (ids, d2) CUDA tensors."""
    torch = _torch()
    ids = ids.contiguous(); d2 = d2.contiguous()
    m = ids.numel()
    kk = min(int(k), m)
    oi = torch.empty(max(kk, 1), dtype=torch.int64, device="cuda")
    od = torch.empty(max(kk, 1), dtype=torch.int64, device="cuda")
    _check(load().spade_knn_topk(ctypes.c_void_p(ids.data_ptr()), ctypes.c_void_p(d2.data_ptr()), m, int(k),
                                 ctypes.c_void_p(oi.data_ptr()), ctypes.c_void_p(od.data_ptr()), _stream(stream)),
           "spade_knn_topk")
    return oi[:kk], od[:kk]


def knn(xy, q, k: int, point_id_base: int = 0, stream=None):
    """The min(k, n) points nearest to q = (qx, qy), ties by id: (ids, d2) int64 CUDA tensors in
    (d2, id) order (spade_knn: all three steps on this device)."""
    torch = _torch()
    xy, n = _points(xy)
    ids = torch.empty(max(int(k), 1), dtype=torch.int64, device="cuda")
    d2 = torch.empty(max(int(k), 1), dtype=torch.int64, device="cuda")
    n_out = ctypes.c_int64()
    _check(load().spade_knn(ctypes.c_void_p(xy.data_ptr()), n, point_id_base, int(q[0]), int(q[1]), int(k),
                            ctypes.c_void_p(ids.data_ptr()), ctypes.c_void_p(d2.data_ptr()), ctypes.byref(n_out),
                            _stream(stream)), "spade_knn")
    return ids[: n_out.value], d2[: n_out.value]
