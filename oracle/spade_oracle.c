/*
 * spade_oracle.c — CPU ORACLE for the SPADE point-in-polygon join (TEST INFRASTRUCTURE ONLY).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library.  It shares no code, header, table or helper with the CUDA path in
 * paper_conf_icde_doraiswamyf22_b200/csrc/ and never includes anything from it.
 *
 * What it computes (brute force over EVERY (point, polygon) pair, no bounding-box filter):
 *
 *   inside(i, p) = XOR over all rings r of polygon p, over all edges (a, b) of r
 *                  (closing edge from the last vertex back to the first included) of
 *                     [ (a.y > py) != (b.y > py) ]  AND  [ b.y > a.y ? o > 0 : o < 0 ],
 *                  o = (b.x - a.x) * (py - a.y) - (b.y - a.y) * (px - a.x)     (exact, __int128)
 *
 *   counts[p] = |{ i : inside(i, p) }|                                  (int64)
 *   pairs     = { (point_id_base + i, p) : inside(i, p) }               sorted by (point, polygon)
 *   select    = { point_id_base + i : exists p with inside(i, p) }      ascending
 *
 * Passages followed (PAPER.md line numbers, /root/reference/PAPER.md):
 *   - selection = objects that satisfy the spatial constraint (ST_INTERSECTS)   P:184 (Sec. 5.2)
 *   - Polygon x Point join = one selection per (layer of) polygons              P:198-200 (Sec. 5.2)
 *   - join output = pairs (x_i, y_j) satisfying the predicate                   P:208 (Sec. 5.2)
 *   - aggregation = per-polygon COUNT of joined points ("plan 2" for points)   P:214 (Sec. 5.2)
 *   - for points, intersection is a containment test                            P:476 (Sec. 7)
 *   - boundary points must be decided exactly ("to enable accuracy")            P:140 (Sec. 4.3)
 *   - polygons may be multi-polygons (rings of one polygon id)                 P:93 footnote
 * Readings where the paper is silent:
 *   C1 half-open even-odd (Franklin pnpoly) tie rule instead of closed ST_INTERSECTS, so that
 *      disjoint tilings assign every point to exactly one polygon; C2 even-odd over all rings;
 *   C3 a point joins every polygon containing it; C9 int64 counts; C10 duplicates counted.
 *
 * The predicate's `b.y > a.y ? o > 0 : o < 0` says: the edge crosses the horizontal line y = py
 * strictly to the right of px (x* - px = o / (b.y - a.y)).  It is the textbook crossing-number
 * test (O'Rourke, Computational Geometry in C, Sec. 7.4) evaluated without rounding.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

/* One edge: does the ray from (px, py) towards +x cross it under the half-open rule? */
static int oracle_edge_crosses(int64_t ax, int64_t ay, int64_t bx, int64_t by, int64_t px, int64_t py) {
    if ((ay > py) == (by > py)) return 0;                 /* does not straddle y = py (half-open) */
    __int128 o = (__int128)(bx - ax) * (py - ay) - (__int128)(by - ay) * (px - ax);
    return by > ay ? (o > 0) : (o < 0);
}

/* inside(point, polygon): parity of crossings over every edge of every ring of the polygon. */
int oracle_point_in_polygon(int64_t px, int64_t py, const int32_t* ring_xy, const int64_t* ring_off,
                            int64_t ring_begin, int64_t ring_end) {
    int parity = 0;
    for (int64_t r = ring_begin; r < ring_end; ++r) {
        int64_t v0 = ring_off[r], v1 = ring_off[r + 1];
        for (int64_t k = v0; k < v1; ++k) {
            int64_t k2 = (k + 1 < v1) ? k + 1 : v0;        /* closing edge back to the first vertex */
            parity ^= oracle_edge_crosses(ring_xy[2 * k], ring_xy[2 * k + 1],
                                          ring_xy[2 * k2], ring_xy[2 * k2 + 1], px, py);
        }
    }
    return parity;
}

/* ------------------------------------------------------------------------------------------ */
/* Brute-force joins, parallel over contiguous point ranges (one plain loop per thread).       */

typedef struct {
    const int32_t* xy; int64_t i0, i1;
    const int32_t* ring_xy; const int64_t* ring_off; const int64_t* poly_ring_off; int32_t num_polys;
    int64_t* counts;                   /* per-thread private counts (num_polys) */
    int64_t* pt; int32_t* pl; int64_t n_pairs, cap_pairs; int oom;   /* per-thread pair buffer */
    int want_pairs;
} oracle_task;

static void* oracle_worker(void* arg) {
    oracle_task* t = (oracle_task*)arg;
    for (int64_t i = t->i0; i < t->i1; ++i) {
        int64_t px = t->xy[2 * i], py = t->xy[2 * i + 1];
        for (int32_t p = 0; p < t->num_polys; ++p) {
            if (!oracle_point_in_polygon(px, py, t->ring_xy, t->ring_off,
                                         t->poly_ring_off[p], t->poly_ring_off[p + 1])) continue;
            if (t->counts) t->counts[p] += 1;
            if (t->want_pairs) {
                if (t->n_pairs == t->cap_pairs) {
                    int64_t nc = t->cap_pairs ? 2 * t->cap_pairs : 1024;
                    int64_t* npt = (int64_t*)realloc(t->pt, nc * sizeof(int64_t));
                    int32_t* npl = (int32_t*)realloc(t->pl, nc * sizeof(int32_t));
                    if (!npt || !npl) { t->oom = 1; if (npt) t->pt = npt; if (npl) t->pl = npl; return NULL; }
                    t->pt = npt; t->pl = npl; t->cap_pairs = nc;
                }
                t->pt[t->n_pairs] = i; t->pl[t->n_pairs] = p; t->n_pairs++;
            }
        }
    }
    return NULL;
}

/* Runs the brute force; returns total pairs (or -1 on allocation failure). If counts != NULL
 * they are OVERWRITTEN with the per-polygon counts.  If want_pairs, up to `capacity` pairs are
 * written in (point, polygon) order; the return value is the total regardless of capacity. */
static int64_t oracle_run(const int32_t* xy, int64_t n, const int32_t* ring_xy, const int64_t* ring_off,
                          const int64_t* poly_ring_off, int32_t num_polys, int nthreads,
                          int64_t* counts, int want_pairs, int64_t point_id_base,
                          int64_t* out_point_ids, int32_t* out_poly_ids, int64_t capacity) {
    if (nthreads < 1) nthreads = 1;
    if (n < nthreads) nthreads = n > 0 ? (int)n : 1;
    oracle_task* tasks = (oracle_task*)calloc(nthreads, sizeof(oracle_task));
    pthread_t* th = (pthread_t*)calloc(nthreads, sizeof(pthread_t));
    if (!tasks || !th) { free(tasks); free(th); return -1; }
    for (int t = 0; t < nthreads; ++t) {
        oracle_task* k = &tasks[t];
        k->xy = xy; k->i0 = n * t / nthreads; k->i1 = n * (t + 1) / nthreads;
        k->ring_xy = ring_xy; k->ring_off = ring_off; k->poly_ring_off = poly_ring_off;
        k->num_polys = num_polys; k->want_pairs = want_pairs;
        k->counts = counts ? (int64_t*)calloc(num_polys > 0 ? num_polys : 1, sizeof(int64_t)) : NULL;
        pthread_create(&th[t], NULL, oracle_worker, k);
    }
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    if (counts) memset(counts, 0, sizeof(int64_t) * (size_t)num_polys);
    int64_t total = 0; int failed = 0;
    for (int t = 0; t < nthreads; ++t) {
        oracle_task* k = &tasks[t];
        if (k->oom) failed = 1;
        if (counts) for (int32_t p = 0; p < num_polys; ++p) counts[p] += k->counts[p];
        for (int64_t q = 0; q < k->n_pairs; ++q, ++total) {
            if (total < capacity) {
                if (out_point_ids) out_point_ids[total] = point_id_base + k->pt[q];
                if (out_poly_ids) out_poly_ids[total] = k->pl[q];
            }
        }
        free(k->counts); free(k->pt); free(k->pl);
    }
    free(tasks); free(th);
    return failed ? -1 : total;
}

/* Per-polygon COUNT of joined points.  counts[num_polys] is overwritten. */
int oracle_join_count(const int32_t* xy, int64_t n, const int32_t* ring_xy, const int64_t* ring_off,
                      const int64_t* poly_ring_off, int32_t num_polys, int64_t* counts, int nthreads) {
    return oracle_run(xy, n, ring_xy, ring_off, poly_ring_off, num_polys, nthreads, counts, 0, 0,
                      NULL, NULL, 0) < 0 ? -1 : 0;
}

/* (point_id, polygon_id) pairs, sorted by point then polygon.
 * Returns the total number of pairs; writes min(total, capacity). */
int64_t oracle_join_pairs(const int32_t* xy, int64_t n, int64_t point_id_base, const int32_t* ring_xy,
                          const int64_t* ring_off, const int64_t* poly_ring_off, int32_t num_polys,
                          int64_t* out_point_ids, int32_t* out_poly_ids, int64_t capacity, int nthreads) {
    return oracle_run(xy, n, ring_xy, ring_off, poly_ring_off, num_polys, nthreads, NULL, 1,
                      point_id_base, out_point_ids, out_poly_ids, capacity);
}

/* Selection: ids of points inside at least one polygon, ascending.  A point inside
 * several polygons is listed once.  Returns the total; writes min(total, capacity). */
int64_t oracle_select(const int32_t* xy, int64_t n, int64_t point_id_base, const int32_t* ring_xy,
                      const int64_t* ring_off, const int64_t* poly_ring_off, int32_t num_polys,
                      int64_t* out_ids, int64_t capacity, int nthreads) {
    int64_t npairs = oracle_run(xy, n, ring_xy, ring_off, poly_ring_off, num_polys, nthreads, NULL, 1,
                                0, NULL, NULL, 0);
    if (npairs < 0) return -1;
    int64_t* pt = (int64_t*)malloc(sizeof(int64_t) * (size_t)(npairs > 0 ? npairs : 1));
    if (!pt) return -1;
    oracle_run(xy, n, ring_xy, ring_off, poly_ring_off, num_polys, nthreads, NULL, 1, 0, pt, NULL, npairs);
    int64_t total = 0;
    for (int64_t q = 0; q < npairs; ++q) {
        if (q > 0 && pt[q] == pt[q - 1]) continue;          /* pairs are grouped by point */
        if (total < capacity) out_ids[total] = point_id_base + pt[q];
        total++;
    }
    free(pt);
    return total;
}
