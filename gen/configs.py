"""The five BASELINE.json configs as concrete, seeded, synthetic workloads.

    c1  10k uniform points on [0,1024)^2 x 16 convex/concave polygons (overlaps, holes)   COUNT
    c2  100M taxi-like points x 1 star query polygon (1,000 vertices, bbox 0.3 x domain) SELECT
    c3  1B taxi-like points x 260 neighbourhood-like tiling polygons (~540 v)            COUNT
    c4  1B taxi-like points x ~2,200 census-like tiling polygons with island holes        PAIRS
    c5  8B points (1B per GPU) x 40k zip-code-like tiling polygons (~1.5k v)             COUNT

Sizes/shapes follow PAPER.md Table 1 (Taxi 1.22B points, Neighborhoods 195 polygons /
538 v avg, Census 2,165 / 72 v, Zip 32,657 / 1,547 v) and the query polygons of P:358 (739 v avg).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import DOMAIN, SgParams, taxi_params, uniform_params
from . import polygons as pg


@dataclass
class Workload:
    name: str
    op: str                    # "count" | "select" | "pairs"
    points: SgParams
    point_seed: int
    n_points: int              # per GPU for the sharded configs
    polys: dict = field(repr=False)
    max_dim: int = 4096        # canvas resolution parameter (C5 reading of DESIGN.md)
    desc: str = ""


def c1(n_points: int = 10_000) -> Workload:
    return Workload("c1_uniform10k_x16poly_1k", "count", uniform_params(0, 0, 1024, 1024), 101, n_points,
                    pg.c1_polygons(102), max_dim=1024,
                    desc="10k uniform points x 16 convex/concave polygons on a 1k x 1k int grid, COUNT")


def c1_edge_points(polys) -> np.ndarray:
    """Test-mode extra points for config 1: every polygon vertex, plus every lattice point on an
    axis-parallel edge and every exact edge midpoint (points exactly on the boundary)."""
    xy = polys["ring_xy"].astype(np.int64)
    ro = polys["ring_off"]
    pts = [xy]
    for r in range(len(ro) - 1):
        ring = xy[ro[r]:ro[r + 1]]
        nxt = np.roll(ring, -1, axis=0)
        for a, b in zip(ring.tolist(), nxt.tolist()):
            if a[0] == b[0]:
                lo, hi = sorted((a[1], b[1]))
                ys = np.arange(lo, hi + 1)
                pts.append(np.stack([np.full_like(ys, a[0]), ys], 1))
            elif a[1] == b[1]:
                lo, hi = sorted((a[0], b[0]))
                xs = np.arange(lo, hi + 1)
                pts.append(np.stack([xs, np.full_like(xs, a[1])], 1))
            if (a[0] + b[0]) % 2 == 0 and (a[1] + b[1]) % 2 == 0:
                pts.append(np.array([[(a[0] + b[0]) // 2, (a[1] + b[1]) // 2]]))
    return np.concatenate(pts).astype(np.int32)


def c2(n_points: int = 100_000_000) -> Workload:
    tp = taxi_params(201)
    rng = np.random.default_rng(202)
    r = 0.15 * DOMAIN
    cx = min(max(tp.cx[0], r), DOMAIN - r)
    cy = min(max(tp.cy[0], r), DOMAIN - r)
    poly = pg.assemble([[pg.star(rng, 1000, cx, cy, r, r, rmin=0.35, smooth=0.01)]])
    return Workload("c2_taxi100M_select_star1000", "select", tp, 201, n_points, poly, max_dim=4096,
                    desc="spatial selection: 100M clustered taxi-like points inside 1 query polygon (1,000 v)")


def c3(n_points: int = 1_000_000_000) -> Workload:
    return Workload("c3_taxi1B_x260_neighborhoods_count", "count", taxi_params(301), 301, n_points,
                    pg.jittered_tiling(20, 13, 135, seed=302), max_dim=16384,
                    desc="point-polygon join COUNT: 1B taxi-like points x 260 neighborhood-like polygons")


def c4(n_points: int = 1_000_000_000) -> Workload:
    return Workload("c4_taxi1B_x2200_census_pairs", "pairs", taxi_params(401), 401, n_points,
                    pg.jittered_tiling(50, 42, 18, n_islands=100, seed=402), max_dim=8192,
                    desc="point-polygon join pairs: 1B points x 2,200 census-tract-like polygons with holes")


def c5(n_points_per_gpu: int = 1_000_000_000) -> Workload:
    return Workload("c5_taxi1Bpergpu_x40k_zip_count", "count", taxi_params(501), 501, n_points_per_gpu,
                    pg.jittered_tiling(200, 200, 375, seed=502), max_dim=16384,
                    desc="scale-out join COUNT: 1B points per GPU x 40k zip-code-like polygons")


# ---- distance-based queries (Sec. 6.4-6.5) ----
# The paper joins the Taxi data with 100..100K random points generated within its extent, at a
# query distance of 5..100 m (20 m by default, Fig. 7).  The synthetic domain [0, 2^24)^2 stands
# for the ~45 km Taxi extent: 1 m = 2^24 / 45,000 grid units.
UNITS_PER_METER = (1 << 24) / 45_000.0


def meters_to_r2(m: float) -> int:
    """Squared radius in grid units for a distance in metres (floor of r^2, reading D2)."""
    r = m * UNITS_PER_METER
    return int(np.floor(r * r))


@dataclass
class DiskWorkload:
    name: str
    op: str                    # "pairs" | "count" | "select" | "knn"
    points: SgParams
    point_seed: int
    n_points: int
    disks: dict = field(repr=False)   # {"center_xy": (D,2) int32, "r2": (D,) int64}
    max_dim: int = 4096
    desc: str = ""
    k: int = 0                 # kNN only
    query: tuple = (0, 0)      # kNN only


def random_centers(n: int, seed: int) -> np.ndarray:
    """n uniform random points within the extent of the taxi-like data (the paper's generated
    point set), kept 1,000 m from the domain edge so every disk stays inside it."""
    rng = np.random.default_rng(seed)
    m = int(1000 * UNITS_PER_METER)
    return rng.integers(m, (1 << 24) - m, size=(n, 2)).astype(np.int32)


def dj(n_points: int = 1_000_000_000, n_disks: int = 100_000, meters: float = 20.0) -> DiskWorkload:
    c = random_centers(n_disks, 602)
    return DiskWorkload(f"dj_taxi1B_x{n_disks // 1000}k_r{int(meters)}m_pairs", "pairs", taxi_params(601), 601,
                        n_points, {"center_xy": c, "r2": np.full(n_disks, meters_to_r2(meters), np.int64)},
                        max_dim=8192,
                        desc=f"type 1 distance join: 1B taxi-like points x {n_disks} random points, distance <= {meters} m")


def dj2(n_points: int = 1_000_000_000, n_disks: int = 100_000) -> DiskWorkload:
    """Type 2 distance join: one radius per generated point, log-uniform in [5, 100] m."""
    c = random_centers(n_disks, 612)
    rng = np.random.default_rng(613)
    m = np.exp(rng.uniform(np.log(5.0), np.log(100.0), n_disks))
    r2 = np.array([meters_to_r2(x) for x in m], np.int64)
    return DiskWorkload(f"dj2_taxi1B_x{n_disks // 1000}k_r5to100m_count", "count", taxi_params(611), 611, n_points,
                        {"center_xy": c, "r2": r2}, max_dim=8192,
                        desc=f"type 2 distance join COUNT: 1B taxi-like points x {n_disks} points with radii 5..100 m")


def knn(n_points: int = 1_000_000_000, k: int = 50) -> DiskWorkload:
    """kNN selection (Fig. 8): the k taxi points nearest to one generated query point."""
    q = random_centers(100, 622)[0]
    return DiskWorkload(f"knn_taxi1B_k{k}", "knn", taxi_params(621), 621, n_points,
                        {"center_xy": np.zeros((0, 2), np.int32), "r2": np.zeros(0, np.int64)}, k=k,
                        query=(int(q[0]), int(q[1])), desc=f"kNN selection: {k} nearest of 1B taxi-like points")


def ov(n_points: int = 1_000_000_000, n_polys: int = 1000) -> Workload:
    """Overlap-heavy polygon set (the layered canvases of P:148 / P:200 and
    the layer index of P:270-274): n_polys concave star query regions (48..160 vertices) centred on
    points drawn from the taxi distribution itself, radii log-uniform in [2^15, 2^20] grid units,
    so the stars pile up over the dense clusters (tens of polygons deep there).  COUNT per
    polygon; a point joins every polygon containing it (reading C3), so sum(counts) = pairs."""
    tp = taxi_params(701)
    rng = np.random.default_rng(702)
    import gen
    ctr = gen.points_host(tp, 703, 0, n_polys).astype(np.int64)
    polys = []
    for i in range(n_polys):
        r = float(2.0 ** rng.uniform(15, 20))
        n = int(rng.integers(48, 161))
        cx = min(max(int(ctr[i, 0]), int(r)), DOMAIN - 1 - int(r))
        cy = min(max(int(ctr[i, 1]), int(r)), DOMAIN - 1 - int(r))
        polys.append([pg.star(rng, n, cx, cy, r, r * rng.uniform(0.5, 1.0), rmin=0.4, smooth=0.05)])
    return Workload(f"ov_taxi1B_x{n_polys // 1000}k_overlapping_stars_count", "count", tp, 701, n_points,
                    pg.assemble(polys), max_dim=8192,
                    desc=f"overlap-heavy join COUNT: 1B taxi-like points x {n_polys} overlapping star polygons")


ALL = {"c1": c1, "c2": c2, "c3": c3, "c4": c4, "c5": c5}
OVERLAP = {"ov": ov}
DISTANCE = {"dj": dj, "dj2": dj2, "knn": knn}


# ---- polygon x polygon join ----------------------------
@dataclass
class PolyJoinWorkload:
    name: str
    op: str                    # "polyjoin"
    polys: dict = field(repr=False)     # D1
    polys2: dict = field(repr=False)    # D2
    max_dim: int = 8192
    desc: str = ""
    n_points: int = 0          # (no point stream)


def pp() -> PolyJoinWorkload:
    """Census-tract-like tiling (C4's 2,200 polygons with island holes) joined with the
    neighbourhood-like tiling (C3's 260 polygons): which tracts meet which neighbourhoods
    (the Polygon x Polygon join of P:202 on Table 1-like data)."""
    return PolyJoinWorkload("pp_census2200_x_neighborhoods260", "polyjoin", c4(1).polys, c3(1).polys, max_dim=8192,
                            desc="polygon x polygon join: 2,200 census-tract-like polygons (holes) x 260 "
                                 "neighbourhood-like polygons, closed-region ST_INTERSECTS")


POLYJOIN = {"pp": pp}
