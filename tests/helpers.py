"""Test-only helpers: small random polygon sets (overlapping, self-intersecting, degenerate)."""
from __future__ import annotations

import numpy as np

from gen import polygons as pg


def random_ring(rng, lo, hi, nmin=2, nmax=12):
    n = int(rng.integers(nmin, nmax + 1))
    kind = rng.random()
    if kind < 0.4:        # arbitrary (self-intersecting) ring
        return np.stack([rng.integers(lo, hi + 1, n), rng.integers(lo, hi + 1, n)], 1)
    if kind < 0.7:        # star around a centre
        c = rng.integers(lo + 2, hi - 1, 2)
        r = max(2, int(rng.integers(2, max(3, (hi - lo) // 2))))
        return np.clip(pg.star(rng, max(3, n), c[0], c[1], r, r, rmin=0.2), lo, hi)
    if kind < 0.85:       # axis-aligned rectangle
        x0, x1 = sorted(rng.integers(lo, hi + 1, 2)); y0, y1 = sorted(rng.integers(lo, hi + 1, 2))
        r = pg.rect(x0, y0, x1, y1)
        return r[::-1] if rng.random() < 0.5 else r
    # rectilinear staircase with repeated / collinear vertices
    pts = [(int(rng.integers(lo, hi + 1)), int(rng.integers(lo, hi + 1)))]
    for _ in range(n):
        x, y = pts[-1]
        if rng.random() < 0.5:
            pts.append((int(rng.integers(lo, hi + 1)), y))
        else:
            pts.append((x, int(rng.integers(lo, hi + 1))))
        if rng.random() < 0.1:
            pts.append(pts[-1])           # zero-length edge
    return np.array(pts, np.int64)


def random_polyset(rng, lo, hi, npoly, max_rings=3):
    polys = []
    for _ in range(npoly):
        polys.append([random_ring(rng, lo, hi) for _ in range(int(rng.integers(1, max_rings + 1)))])
    return pg.assemble(polys)


def lattice(x0, y0, x1, y1):
    xs, ys = np.meshgrid(np.arange(x0, x1 + 1), np.arange(y0, y1 + 1))
    return np.stack([xs.ravel(), ys.ravel()], 1).astype(np.int32)


def sorted_pairs(pt, pl):
    pt = np.asarray(pt, np.int64); pl = np.asarray(pl, np.int64)
    o = np.lexsort((pl, pt))
    return pt[o], pl[o]


def valid_polyset(rng, n, lo, hi, scale=1):
    """Valid polygons (simple rings, no zero-length edges): stars, rectangles, rectangles with a
    rectangular hole, two-component rectangles."""
    polys = []
    for _ in range(n):
        kind = rng.random()
        cx, cy = rng.integers(lo + 6, hi - 5, 2)
        if kind < 0.4:
            r = pg.star(rng, int(rng.integers(3, 9)), cx, cy, rng.integers(3, 8), rng.integers(3, 8), rmin=0.5)
            r = r[np.any(r != np.roll(r, 1, 0), axis=1)]
            if len(r) < 3:
                r = pg.rect(cx - 2, cy - 2, cx + 2, cy + 2)
            polys.append([r])
        else:
            w, h = rng.integers(2, 8, 2)
            outer = pg.rect(cx - w, cy - h, cx + w, cy + h)
            if kind < 0.6 and w >= 4 and h >= 4:
                polys.append([outer, pg.rect(cx - w + 2, cy - h + 2, cx + w - 2, cy + h - 2)])
            elif kind < 0.8:
                polys.append([outer, pg.rect(cx + w + 2, cy, cx + w + 4, cy + 3)])
            else:
                polys.append([outer])
    out = pg.assemble(polys)
    out["ring_xy"] = (np.asarray(out["ring_xy"], np.int64) * scale).astype(np.int32)
    return out
