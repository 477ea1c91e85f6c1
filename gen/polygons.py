"""Seeded synthetic POLYGON sets (input data only; numpy, host).

A polygon set is a dict of int arrays, the layout the C ABI takes (include/spade.h):
    ring_xy       int32 (V, 2)  vertices of every ring, rings implicitly closed
    ring_off      int64 (R+1)   ring r = vertices [ring_off[r], ring_off[r+1])
    poly_ring_off int64 (P+1)   polygon p = rings [poly_ring_off[p], poly_ring_off[p+1])

Shapes mimic the paper's polygon data sets (Table 1): neighbourhood / census
tract / zip-code like tilings (shared wiggly borders, island holes), star-shaped query polygons
(~739 vertices on average for the Taxi selection constraints) and rectangle "parcels"
(non-intersecting rectangles).
"""
from __future__ import annotations

import numpy as np


def assemble(polys) -> dict:
    """polys: list of polygons, each a list of rings, each an (k, 2) integer array."""
    rings, ring_off, poly_ring_off = [], [0], [0]
    for rs in polys:
        for r in rs:
            r = np.asarray(r, dtype=np.int64).reshape(-1, 2)
            rings.append(r)
            ring_off.append(ring_off[-1] + len(r))
        poly_ring_off.append(len(ring_off) - 1)
    xy = np.concatenate(rings) if rings else np.zeros((0, 2), np.int64)
    assert xy.size == 0 or (xy.min() >= -(1 << 30) and xy.max() < (1 << 30))
    return {"ring_xy": xy.astype(np.int32), "ring_off": np.asarray(ring_off, np.int64),
            "poly_ring_off": np.asarray(poly_ring_off, np.int64)}


def concat_sets(*sets) -> dict:
    """Polygon ids of later sets follow those of earlier ones."""
    polys = []
    for s in sets:
        polys += polygons_as_lists(s)
    return assemble(polys)


def polygons_as_lists(s) -> list:
    out = []
    xy, ro, pro = s["ring_xy"], s["ring_off"], s["poly_ring_off"]
    for p in range(len(pro) - 1):
        out.append([xy[ro[r]:ro[r + 1]].astype(np.int64) for r in range(pro[p], pro[p + 1])])
    return out


def rect(x0, y0, x1, y1):
    return np.array([[x0, y0], [x1, y0], [x1, y1], [x0, y1]], dtype=np.int64)


def grid_tiling(nx, ny, x0, y0, cw, ch) -> dict:
    """nx*ny axis-aligned rectangles; polygon id = j*nx + i covers [x0+i*cw, x0+(i+1)*cw) x ..."""
    return assemble([[rect(x0 + i * cw, y0 + j * ch, x0 + (i + 1) * cw, y0 + (j + 1) * ch)]
                     for j in range(ny) for i in range(nx)])


def star(rng, n, cx, cy, rx, ry, rmin=0.45, smooth=0.0):
    """Star-shaped (generally concave) ring: n vertices at angles 2*pi*k/n, random radii."""
    th = 2 * np.pi * np.arange(n) / n
    u = rng.uniform(rmin, 1.0, n)
    if smooth > 0:   # low-pass the radii for a more realistic outline
        k = max(1, int(smooth * n))
        u = np.convolve(np.concatenate([u[-k:], u, u[:k]]), np.ones(2 * k + 1) / (2 * k + 1), "same")[k:-k]
    x = np.rint(cx + rx * u * np.cos(th)).astype(np.int64)
    y = np.rint(cy + ry * u * np.sin(th)).astype(np.int64)
    return np.stack([x, y], 1)


def convex_hull(pts):
    """Monotone-chain hull of integer points (exact integer orientation), CCW, no repeats."""
    p = sorted(set(map(tuple, np.asarray(pts, np.int64).tolist())))
    if len(p) <= 2:
        return np.array(p, np.int64)

    def cross(o, a, b):
        return (a[0] - o[0]) * (b[1] - o[1]) - (a[1] - o[1]) * (b[0] - o[0])
    lo, hi = [], []
    for q in p:
        while len(lo) >= 2 and cross(lo[-2], lo[-1], q) <= 0:
            lo.pop()
        lo.append(q)
    for q in reversed(p):
        while len(hi) >= 2 and cross(hi[-2], hi[-1], q) <= 0:
            hi.pop()
        hi.append(q)
    return np.array(lo[:-1] + hi[:-1], np.int64)


def _with_degeneracies(rng, ring):
    """Add axis-parallel runs and collinear midpoints to a ring (edge cases for the tie rule)."""
    r = [tuple(v) for v in ring.tolist()]
    out = []
    for k, v in enumerate(r):
        out.append(v)
        w = r[(k + 1) % len(r)]
        c = rng.random()
        if c < 0.25:                                  # axis-parallel detour: v -> (w.x, v.y) -> w
            out.append((w[0], v[1]))
        elif c < 0.45 and (v[0] + w[0]) % 2 == 0 and (v[1] + w[1]) % 2 == 0:
            out.append(((v[0] + w[0]) // 2, (v[1] + w[1]) // 2))   # exact collinear midpoint
    return np.array(out, np.int64)


def c1_polygons(seed: int = 102, size: int = 1024) -> dict:
    """Config 1: 16 convex/concave polygons on a size x size integer grid, overlaps allowed:
    8 convex hulls of 6-20 lattice points, 6 stars (8-40 vertices) with axis-parallel and collinear
    runs, 2 polygons with a hole."""
    rng = np.random.default_rng(seed)
    polys = []
    for _ in range(8):
        w = int(rng.integers(80, 400)); h = int(rng.integers(80, 400))
        x0 = int(rng.integers(0, size - w)); y0 = int(rng.integers(0, size - h))
        pts = np.stack([rng.integers(x0, x0 + w, 20), rng.integers(y0, y0 + h, 20)], 1)[: int(rng.integers(6, 21))]
        hull = convex_hull(pts)
        if len(hull) < 3:
            hull = rect(x0, y0, x0 + w, y0 + h)
        polys.append([hull])
    for _ in range(6):
        r = int(rng.integers(60, 220))
        cx = int(rng.integers(r, size - r)); cy = int(rng.integers(r, size - r))
        s = star(rng, int(rng.integers(8, 41)), cx, cy, r, r)
        polys.append([_with_degeneracies(rng, s)])
    for _ in range(2):
        r = int(rng.integers(120, 240))
        cx = int(rng.integers(r, size - r)); cy = int(rng.integers(r, size - r))
        outer = star(rng, int(rng.integers(10, 30)), cx, cy, r, r, rmin=0.75)
        hole = star(rng, int(rng.integers(6, 16)), cx, cy, r * 0.4, r * 0.4, rmin=0.6)[::-1]
        polys.append([outer, hole])
    return assemble(polys)


def _wiggle(rng, shape, k):
    """Smooth random profile in [-1, 1] for k interior vertices of each side (two sinusoids +
    small noise), tapered to 0 at both ends by 4t(1-t)."""
    t = np.arange(1, k + 1) / (k + 1)
    f1 = rng.integers(1, 4, shape)[..., None]
    f2 = rng.integers(2, 7, shape)[..., None]
    p1 = rng.uniform(0, 2 * np.pi, shape)[..., None]
    p2 = rng.uniform(0, 2 * np.pi, shape)[..., None]
    prof = 0.6 * np.sin(2 * np.pi * f1 * t + p1) + 0.3 * np.sin(2 * np.pi * f2 * t + p2)
    prof = prof + 0.1 * rng.uniform(-1, 1, tuple(shape) + (k,))
    return prof * (4 * t * (1 - t))


def jittered_tiling(nx, ny, vps, domain=1 << 24, jitter=0.08, wiggle=0.08, n_islands=0, seed=0) -> dict:
    """Exact planar partition of [0, domain]^2 into nx*ny cells with wiggly shared borders.

    Corners form a jittered lattice (border corners stay on the border); each lattice side is a
    polyline with vps-1 interior vertices displaced perpendicular to the side by a tapered smooth
    profile (amplitude <= wiggle * cell); sides on the domain border are straight (collinear
    vertices).  Each side is stored once and used reversed by the neighbouring cell, so cells
    share their borders vertex for vertex.  Cell (i, j) has polygon id j*nx + i and 4*vps vertices.
    n_islands random cells get a star-shaped island: a hole ring of the host cell and a polygon of
    its own (ids nx*ny ...).
    """
    rng = np.random.default_rng(seed)
    k = vps - 1
    X = np.rint(np.arange(nx + 1) * domain / nx).astype(np.float64)
    Y = np.rint(np.arange(ny + 1) * domain / ny).astype(np.float64)
    cw, ch = domain / nx, domain / ny
    cx = np.broadcast_to(X[None, :], (ny + 1, nx + 1)).copy()
    cy = np.broadcast_to(Y[:, None], (ny + 1, nx + 1)).copy()
    jx = rng.uniform(-jitter, jitter, cx.shape) * cw
    jy = rng.uniform(-jitter, jitter, cy.shape) * ch
    jx[:, 0] = jx[:, -1] = 0
    jy[0, :] = jy[-1, :] = 0
    cx += jx
    cy += jy
    cx = np.rint(cx)
    cy = np.rint(cy)
    t = (np.arange(1, k + 1) / (k + 1)) if k > 0 else np.zeros(0)
    # horizontal sides H[j, i]: corner (i, j) -> (i+1, j); displaced in y
    hx = cx[:, :-1, None] + (cx[:, 1:, None] - cx[:, :-1, None]) * t
    hy = cy[:, :-1, None] + (cy[:, 1:, None] - cy[:, :-1, None]) * t
    if k > 0:
        hw = _wiggle(rng, (ny + 1, nx), k) * wiggle * ch
        hw[0] = hw[-1] = 0
        hy = hy + hw
    # vertical sides V[j, i]: corner (i, j) -> (i, j+1); displaced in x
    vx = cx[:-1, :, None] + (cx[1:, :, None] - cx[:-1, :, None]) * t
    vy = cy[:-1, :, None] + (cy[1:, :, None] - cy[:-1, :, None]) * t
    if k > 0:
        vw = _wiggle(rng, (ny, nx + 1), k) * wiggle * cw
        vw[:, 0] = vw[:, -1] = 0
        vx = vx + vw
    H = np.stack([np.rint(hx), np.rint(hy)], -1).astype(np.int64)   # (ny+1, nx, k, 2)
    V = np.stack([np.rint(vx), np.rint(vy)], -1).astype(np.int64)   # (ny, nx+1, k, 2)
    C = np.stack([cx, cy], -1).astype(np.int64)                      # (ny+1, nx+1, 2)
    # ring of cell (i, j): c(i,j), H[j,i], c(i+1,j), V[j,i+1], c(i+1,j+1), rev H[j+1,i], c(i,j+1), rev V[j,i]
    ring = np.concatenate([
        C[:-1, :-1, None], H[:-1],
        C[:-1, 1:, None], V[:, 1:],
        C[1:, 1:, None], H[1:, :, ::-1],
        C[1:, :-1, None], V[:, :-1, ::-1],
    ], axis=2)                                                       # (ny, nx, 4*vps, 2)
    ncell = nx * ny
    ring_xy = ring.reshape(ncell * 4 * vps, 2)
    ring_off = np.arange(ncell + 1, dtype=np.int64) * (4 * vps)
    if n_islands == 0:
        return {"ring_xy": ring_xy.astype(np.int32), "ring_off": ring_off,
                "poly_ring_off": np.arange(ncell + 1, dtype=np.int64)}
    hosts = np.sort(rng.choice(ncell, size=n_islands, replace=False))
    isl = []
    for h in hosts:
        j, i = divmod(int(h), nx)
        ccx = C[j:j + 2, i:i + 2, 0].mean()
        ccy = C[j:j + 2, i:i + 2, 1].mean()
        r = 0.15 * min(cw, ch)
        isl.append(star(rng, max(8, 2 * vps), ccx, ccy, r, r, rmin=0.5, smooth=0.05))
    # rings: cells (hosts get their hole ring right after their outer ring), then islands
    rings, polys_rings = [], []
    host_set = {int(h): q for q, h in enumerate(hosts)}
    for c in range(ncell):
        rs = [ring_xy[c * 4 * vps:(c + 1) * 4 * vps]]
        if c in host_set:
            rs.append(isl[host_set[c]][::-1])
        polys_rings.append(rs)
    for q in range(n_islands):
        polys_rings.append([isl[q]])
    return assemble(polys_rings)


def guillotine_parcels(rng, n, x0, y0, x1, y1, min_size=2):
    """Recursive guillotine split of [x0,x1) x [y0,y1) into <= n axis-aligned parcels ("parcels",
    P:448).  Returns (rects list [(x0,y0,x1,y1)], tree) where tree is a kd structure used by tests to
    label points WITHOUT any point-in-polygon arithmetic (half-open intervals)."""
    rects = []

    def split(bx0, by0, bx1, by1, m):
        if m <= 1 or (bx1 - bx0 < 2 * min_size and by1 - by0 < 2 * min_size):
            rects.append((bx0, by0, bx1, by1))
            return ("leaf", len(rects) - 1)
        m1 = m // 2
        if (bx1 - bx0 >= by1 - by0 and bx1 - bx0 >= 2 * min_size) or by1 - by0 < 2 * min_size:
            s = int(rng.integers(bx0 + min_size, bx1 - min_size + 1))
            return ("x", s, split(bx0, by0, s, by1, m1), split(s, by0, bx1, by1, m - m1))
        s = int(rng.integers(by0 + min_size, by1 - min_size + 1))
        return ("y", s, split(bx0, by0, bx1, s, m1), split(bx0, s, bx1, by1, m - m1))

    tree = split(x0, y0, x1, y1, n)
    return rects, tree


def kd_label(tree, x, y):
    while tree[0] != "leaf":
        axis, s, lo, hi = tree
        tree = lo if (x if axis == "x" else y) < s else hi
    return tree[1]
