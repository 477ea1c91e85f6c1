"""CPU oracle for the SPADE point-in-polygon join — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_icde_doraiswamyf22_b200``) never imports it and shares no code with it.

The arithmetic lives in ``spade_oracle.c`` (brute force over every (point, polygon) pair,
half-open even-odd rule, ``__int128`` cross products); see its header for the definition and
the PAPER.md passages it follows.  This module
is argument marshalling (numpy -> ctypes) only.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile spade_oracle.c (+ the R-tree CPU baseline, rtree_join.c) into liboracle.so
    (plain gcc, -O2, pthreads)."""
    srcs = [os.path.join(_HERE, "spade_oracle.c"), os.path.join(_HERE, "rtree_join.c"),
            os.path.join(_HERE, "distance_oracle.c"), os.path.join(_HERE, "polygon_join_oracle.c")]
    newest = max(os.path.getmtime(x) for x in srcs)
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < newest:
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread", "-o", _LIB_PATH, *srcs])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        P = ctypes.c_void_p
        i64, i32 = ctypes.c_int64, ctypes.c_int32
        lib.oracle_point_in_polygon.argtypes = [i64, i64, P, P, i64, i64]
        lib.oracle_point_in_polygon.restype = ctypes.c_int
        lib.oracle_join_count.argtypes = [P, i64, P, P, P, i32, P, ctypes.c_int]
        lib.oracle_join_count.restype = ctypes.c_int
        lib.oracle_join_pairs.argtypes = [P, i64, i64, P, P, P, i32, P, P, i64, ctypes.c_int]
        lib.oracle_join_pairs.restype = i64
        lib.oracle_select.argtypes = [P, i64, i64, P, P, P, i32, P, i64, ctypes.c_int]
        lib.oracle_select.restype = i64
        lib.rtree_join_count.argtypes = [P, i64, P, P, P, i32, P, ctypes.c_int]
        lib.rtree_join_count.restype = ctypes.c_int
        lib.oracle_in_disk.argtypes = [i64, i64, i64, i64, i64]
        lib.oracle_in_disk.restype = ctypes.c_int
        lib.oracle_disk_join_count.argtypes = [P, i64, P, P, i32, P, ctypes.c_int]
        lib.oracle_disk_join_count.restype = ctypes.c_int
        lib.oracle_disk_join_pairs.argtypes = [P, i64, i64, P, P, i32, P, P, i64, ctypes.c_int]
        lib.oracle_disk_join_pairs.restype = i64
        lib.oracle_disk_select.argtypes = [P, i64, i64, P, P, i32, P, i64, ctypes.c_int]
        lib.oracle_disk_select.restype = i64
        lib.oracle_segments_intersect.argtypes = [i64] * 8
        lib.oracle_segments_intersect.restype = ctypes.c_int
        lib.oracle_polygons_intersect.argtypes = [P, P, P, i32, P, P, P, i32]
        lib.oracle_polygons_intersect.restype = ctypes.c_int
        lib.oracle_polygon_join.argtypes = [P, P, P, i32, P, P, P, i32, P, P, i64, ctypes.c_int]
        lib.oracle_polygon_join.restype = i64
        lib.oracle_knn.argtypes = [P, i64, i64, i64, i64, i64, P, P]
        lib.oracle_knn.restype = i64
        _lib = lib
    return _lib


def default_threads() -> int:
    return len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)


def _polys(polys):
    ring_xy = np.ascontiguousarray(polys["ring_xy"], dtype=np.int32).reshape(-1, 2)
    ring_off = np.ascontiguousarray(polys["ring_off"], dtype=np.int64)
    poly_ring_off = np.ascontiguousarray(polys["poly_ring_off"], dtype=np.int64)
    return ring_xy, ring_off, poly_ring_off, len(poly_ring_off) - 1


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def point_in_polygon(px: int, py: int, polys, p: int) -> bool:
    """inside(point, polygon p) under the half-open even-odd rule."""
    lib = _load()
    ring_xy, ring_off, poly_ring_off, _ = _polys(polys)
    return bool(lib.oracle_point_in_polygon(int(px), int(py), _ptr(ring_xy), _ptr(ring_off),
                                            int(poly_ring_off[p]), int(poly_ring_off[p + 1])))


def join_count(xy, polys, nthreads: int | None = None) -> np.ndarray:
    """int64[P] per-polygon counts."""
    lib = _load()
    xy = np.ascontiguousarray(xy, dtype=np.int32).reshape(-1, 2)
    ring_xy, ring_off, poly_ring_off, P = _polys(polys)
    counts = np.zeros(max(P, 1), dtype=np.int64)
    rc = lib.oracle_join_count(_ptr(xy), len(xy), _ptr(ring_xy), _ptr(ring_off), _ptr(poly_ring_off), P,
                               _ptr(counts), nthreads or default_threads())
    if rc != 0:
        raise MemoryError("oracle_join_count failed")
    return counts[:P]


def join_pairs(xy, polys, point_id_base: int = 0, nthreads: int | None = None):
    """(point_ids int64[M], poly_ids int32[M]) sorted by (point, polygon)."""
    lib = _load()
    xy = np.ascontiguousarray(xy, dtype=np.int32).reshape(-1, 2)
    ring_xy, ring_off, poly_ring_off, P = _polys(polys)
    nt = nthreads or default_threads()
    total = lib.oracle_join_pairs(_ptr(xy), len(xy), point_id_base, _ptr(ring_xy), _ptr(ring_off),
                                  _ptr(poly_ring_off), P, None, None, 0, nt)
    if total < 0:
        raise MemoryError("oracle_join_pairs failed")
    pt = np.empty(max(total, 1), dtype=np.int64)
    pl = np.empty(max(total, 1), dtype=np.int32)
    lib.oracle_join_pairs(_ptr(xy), len(xy), point_id_base, _ptr(ring_xy), _ptr(ring_off),
                          _ptr(poly_ring_off), P, _ptr(pt), _ptr(pl), total, nt)
    return pt[:total], pl[:total]


def select(xy, polys, point_id_base: int = 0, nthreads: int | None = None) -> np.ndarray:
    """int64 ids of points inside at least one polygon, ascending."""
    lib = _load()
    xy = np.ascontiguousarray(xy, dtype=np.int32).reshape(-1, 2)
    ring_xy, ring_off, poly_ring_off, P = _polys(polys)
    nt = nthreads or default_threads()
    out = np.empty(max(len(xy), 1), dtype=np.int64)
    total = lib.oracle_select(_ptr(xy), len(xy), point_id_base, _ptr(ring_xy), _ptr(ring_off),
                              _ptr(poly_ring_off), P, _ptr(out), len(out), nt)
    if total < 0:
        raise MemoryError("oracle_select failed")
    return out[:total]


def rtree_join_count(xy, polys, nthreads: int | None = None) -> np.ndarray:
    """COUNT by the simple R-tree CPU join (STR over polygon bboxes + the same exact predicate);
    the second CPU baseline of BASELINE.json's north_star.  Identical results to join_count."""
    lib = _load()
    xy = np.ascontiguousarray(xy, dtype=np.int32).reshape(-1, 2)
    ring_xy, ring_off, poly_ring_off, P = _polys(polys)
    counts = np.zeros(max(P, 1), dtype=np.int64)
    rc = lib.rtree_join_count(_ptr(xy), len(xy), _ptr(ring_xy), _ptr(ring_off), _ptr(poly_ring_off), P,
                              _ptr(counts), nthreads or default_threads())
    if rc != 0:
        raise MemoryError("rtree_join_count failed")
    return counts[:P]


def labels_at(xy, polys, nthreads: int | None = None):
    """For each point, the sorted list of polygons containing it (via join_pairs)."""
    pt, pl = join_pairs(xy, polys, 0, nthreads)
    n = len(np.asarray(xy).reshape(-1, 2))
    out = [[] for _ in range(n)]
    for a, b in zip(pt.tolist(), pl.tolist()):
        out[a].append(b)
    return out


# ---- distance-based queries over points and kNN (distance_oracle.c) ----

def _disks(disks):
    cxy = np.ascontiguousarray(disks["center_xy"], dtype=np.int32).reshape(-1, 2)
    r2 = np.ascontiguousarray(disks["r2"], dtype=np.int64).reshape(-1)
    assert len(r2) == len(cxy)
    return cxy, r2, len(cxy)


def in_disk(px: int, py: int, cx: int, cy: int, r2: int) -> bool:
    """(px-cx)^2 + (py-cy)^2 <= r2 (closed disk, squared integer radius)."""
    return bool(_load().oracle_in_disk(int(px), int(py), int(cx), int(cy), int(r2)))


def disk_join_count(xy, disks, nthreads: int | None = None) -> np.ndarray:
    """int64[D] number of points within each disk (aggregation over a distance canvas)."""
    lib = _load()
    xy = np.ascontiguousarray(xy, dtype=np.int32).reshape(-1, 2)
    cxy, r2, D = _disks(disks)
    counts = np.zeros(max(D, 1), dtype=np.int64)
    if lib.oracle_disk_join_count(_ptr(xy), len(xy), _ptr(cxy), _ptr(r2), D, _ptr(counts),
                                  nthreads or default_threads()) != 0:
        raise MemoryError("oracle_disk_join_count failed")
    return counts[:D]


def disk_join_pairs(xy, disks, point_id_base: int = 0, nthreads: int | None = None):
    """(point_ids int64, disk_ids int32) sorted by (point, disk): the type 1 / type 2 distance
    join with the disks as the constraint side."""
    lib = _load()
    xy = np.ascontiguousarray(xy, dtype=np.int32).reshape(-1, 2)
    cxy, r2, D = _disks(disks)
    nt = nthreads or default_threads()
    total = lib.oracle_disk_join_pairs(_ptr(xy), len(xy), point_id_base, _ptr(cxy), _ptr(r2), D, None, None, 0, nt)
    if total < 0:
        raise MemoryError("oracle_disk_join_pairs failed")
    pt = np.empty(max(total, 1), dtype=np.int64)
    pl = np.empty(max(total, 1), dtype=np.int32)
    lib.oracle_disk_join_pairs(_ptr(xy), len(xy), point_id_base, _ptr(cxy), _ptr(r2), D, _ptr(pt), _ptr(pl), total, nt)
    return pt[:total], pl[:total]


def disk_select(xy, disks, point_id_base: int = 0, nthreads: int | None = None) -> np.ndarray:
    """int64 ids of points within at least one disk, ascending (distance selection)."""
    lib = _load()
    xy = np.ascontiguousarray(xy, dtype=np.int32).reshape(-1, 2)
    cxy, r2, D = _disks(disks)
    out = np.empty(max(len(xy), 1), dtype=np.int64)
    total = lib.oracle_disk_select(_ptr(xy), len(xy), point_id_base, _ptr(cxy), _ptr(r2), D, _ptr(out), len(out),
                                   nthreads or default_threads())
    if total < 0:
        raise MemoryError("oracle_disk_select failed")
    return out[:total]


def knn(xy, q, k: int, point_id_base: int = 0):
    """(ids int64[min(k,n)], dist2 int64) of the k points nearest to q, ties by id."""
    lib = _load()
    xy = np.ascontiguousarray(xy, dtype=np.int32).reshape(-1, 2)
    m = max(min(k, len(xy)), 1)
    ids = np.empty(m, dtype=np.int64)
    d2 = np.empty(m, dtype=np.int64)
    got = lib.oracle_knn(_ptr(xy), len(xy), point_id_base, int(q[0]), int(q[1]), int(k), _ptr(ids), _ptr(d2))
    if got < 0:
        raise MemoryError("oracle_knn failed")
    return ids[:got], d2[:got]


# ---- polygon x polygon join (polygon_join_oracle.c, reading C15) ----------------

def segments_intersect(a, b, c, d) -> bool:
    """Closed segments a-b and c-d share a point (textbook SEGMENTS-INTERSECT, exact)."""
    return bool(_load().oracle_segments_intersect(int(a[0]), int(a[1]), int(b[0]), int(b[1]),
                                                   int(c[0]), int(c[1]), int(d[0]), int(d[1])))


def polygons_intersect(polys1, a: int, polys2, b: int) -> bool:
    """Closed regions of polygon a of polys1 and polygon b of polys2 intersect (ST_INTERSECTS)."""
    x1, r1, p1, _ = _polys(polys1)
    x2, r2, p2, _ = _polys(polys2)
    return bool(_load().oracle_polygons_intersect(_ptr(x1), _ptr(r1), _ptr(p1), int(a), _ptr(x2), _ptr(r2), _ptr(p2), int(b)))


def polygon_join(polys1, polys2, nthreads: int | None = None):
    """All (a, b) with polygon a of polys1 intersecting polygon b of polys2 (closed regions),
    sorted by (a, b): two int32 arrays.  Brute force over every polygon pair and edge pair."""
    lib = _load()
    x1, r1, p1, n1 = _polys(polys1)
    x2, r2, p2, n2 = _polys(polys2)
    nt = nthreads or default_threads()
    cap = 1024
    while True:
        a = np.empty(cap, np.int32)
        b = np.empty(cap, np.int32)
        tot = lib.oracle_polygon_join(_ptr(x1), _ptr(r1), _ptr(p1), n1, _ptr(x2), _ptr(r2), _ptr(p2), n2,
                                      _ptr(a), _ptr(b), cap, nt)
        if tot < 0:
            raise MemoryError("oracle_polygon_join")
        if tot <= cap:
            return a[:tot], b[:tot]
        cap = int(tot)
