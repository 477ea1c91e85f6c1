/*
 * polygon_join_oracle.c — CPU ORACLE for the polygon x polygon join (TEST INFRASTRUCTURE ONLY).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library.  It shares no code, header, table or helper with the CUDA path in
 * paper_conf_icde_doraiswamyf22_b200/csrc/ (it calls only oracle_point_in_polygon of
 * spade_oracle.c, the oracle's own point test).
 *
 * What it computes (brute force over EVERY (polygon of D1, polygon of D2) pair and, for each,
 * over EVERY (edge of A, edge of B) pair; no bounding-box filter):
 *
 *   join = { (a, b) : intersects(A_a, B_b) },  sorted by (a, b), where
 *   intersects(A, B) =  some edge of A and some edge of B intersect as CLOSED segments
 *                    OR the first vertex of some ring of B is inside A
 *                    OR the first vertex of some ring of A is inside B
 *   (edges: every ring's consecutive vertices plus the closing edge; "inside": the half-open
 *    even-odd rule of spade_oracle.c, oracle_point_in_polygon).
 *
 * Why this is ST_INTERSECTS of the closed regions (reading C15): if the boundaries of A
 * and B share a point, the closed regions intersect (the first clause).  If they share none, the
 * closed regions intersect iff one contains a point of the other, and then the boundary of a
 * connected component of their intersection lies on one polygon's boundary only, i.e. a whole
 * ring of one polygon lies in the other -- so that ring's first vertex is inside it, and, being
 * on no edge of the other polygon, the half-open test decides it exactly.
 *
 * Closed segment intersection: the textbook test (Cormen et al., Introduction to Algorithms,
 * SEGMENTS-INTERSECT, Sec. 33.1): the segments intersect iff each straddles the other's line,
 * or an endpoint of one is collinear with and within the other.  Orientations in __int128.
 *
 * Domain: valid polygons (each ring has >= 3 vertices, no zero-length edges, no polygon uses a
 * segment twice or along overlapping collinear edges); rings may touch at points, polygons may
 * have holes and several outer rings, different polygons may share edges.
 *
 * Passages followed: Polygon x Polygon join as selections over one data set's
 * polygons P:202 (Sec. 5.2); the spatial constraint is ST_INTERSECTS P:184; polygon-polygon
 * intersection tests on boundary pixels P:140, P:146 (Sec. 4.3).
 */
#include <stdint.h>
#include <stdlib.h>
#include <pthread.h>

int oracle_point_in_polygon(int64_t px, int64_t py, const int32_t* ring_xy, const int64_t* ring_off,
                            int64_t ring_begin, int64_t ring_end);

/* sign of the cross product (q - p) x (r - p) */
static int orient(int64_t px, int64_t py, int64_t qx, int64_t qy, int64_t rx, int64_t ry) {
    __int128 v = (__int128)(qx - px) * (ry - py) - (__int128)(qy - py) * (rx - px);
    return v > 0 ? 1 : (v < 0 ? -1 : 0);
}

/* r collinear with p-q: is r within the segment's bounding box? */
static int on_segment(int64_t px, int64_t py, int64_t qx, int64_t qy, int64_t rx, int64_t ry) {
    return (rx >= (px < qx ? px : qx)) && (rx <= (px > qx ? px : qx)) &&
           (ry >= (py < qy ? py : qy)) && (ry <= (py > qy ? py : qy));
}

int oracle_segments_intersect(int64_t ax, int64_t ay, int64_t bx, int64_t by,
                              int64_t cx, int64_t cy, int64_t dx, int64_t dy) {
    int d1 = orient(cx, cy, dx, dy, ax, ay), d2 = orient(cx, cy, dx, dy, bx, by);
    int d3 = orient(ax, ay, bx, by, cx, cy), d4 = orient(ax, ay, bx, by, dx, dy);
    if (d1 * d2 < 0 && d3 * d4 < 0) return 1;
    if (d1 == 0 && on_segment(cx, cy, dx, dy, ax, ay)) return 1;
    if (d2 == 0 && on_segment(cx, cy, dx, dy, bx, by)) return 1;
    if (d3 == 0 && on_segment(ax, ay, bx, by, cx, cy)) return 1;
    if (d4 == 0 && on_segment(ax, ay, bx, by, dx, dy)) return 1;
    return 0;
}

typedef struct { const int32_t* xy; const int64_t* ro; const int64_t* pro; int32_t n; } pset;

static int edge_contact(const pset* A, int32_t a, const pset* B, int32_t b) {
    for (int64_t r = A->pro[a]; r < A->pro[a + 1]; ++r)
        for (int64_t k = A->ro[r]; k < A->ro[r + 1]; ++k) {
            int64_t k2 = k + 1 < A->ro[r + 1] ? k + 1 : A->ro[r];
            for (int64_t s = B->pro[b]; s < B->pro[b + 1]; ++s)
                for (int64_t m = B->ro[s]; m < B->ro[s + 1]; ++m) {
                    int64_t m2 = m + 1 < B->ro[s + 1] ? m + 1 : B->ro[s];
                    if (oracle_segments_intersect(A->xy[2 * k], A->xy[2 * k + 1], A->xy[2 * k2], A->xy[2 * k2 + 1],
                                                  B->xy[2 * m], B->xy[2 * m + 1], B->xy[2 * m2], B->xy[2 * m2 + 1]))
                        return 1;
                }
        }
    return 0;
}

/* the first vertex of some ring of Q inside polygon p of P */
static int ring_vertex_inside(const pset* Q, int32_t q, const pset* P, int32_t p) {
    for (int64_t r = Q->pro[q]; r < Q->pro[q + 1]; ++r) {
        if (Q->ro[r + 1] <= Q->ro[r]) continue;
        int64_t v = Q->ro[r];
        if (oracle_point_in_polygon(Q->xy[2 * v], Q->xy[2 * v + 1], P->xy, P->ro, P->pro[p], P->pro[p + 1])) return 1;
    }
    return 0;
}

int oracle_polygons_intersect(const int32_t* xy1, const int64_t* ro1, const int64_t* pro1, int32_t a,
                              const int32_t* xy2, const int64_t* ro2, const int64_t* pro2, int32_t b) {
    pset A = {xy1, ro1, pro1, 0}, B = {xy2, ro2, pro2, 0};
    return edge_contact(&A, a, &B, b) || ring_vertex_inside(&B, b, &A, a) || ring_vertex_inside(&A, a, &B, b);
}

typedef struct { pset A, B; int32_t a0, a1; uint8_t* hit; } pj_task;

static void* pj_worker(void* arg) {
    pj_task* t = (pj_task*)arg;
    for (int32_t a = t->a0; a < t->a1; ++a)
        for (int32_t b = 0; b < t->B.n; ++b)
            t->hit[(int64_t)a * t->B.n + b] = (uint8_t)(edge_contact(&t->A, a, &t->B, b) ||
                                                        ring_vertex_inside(&t->B, b, &t->A, a) ||
                                                        ring_vertex_inside(&t->A, a, &t->B, b));
    return NULL;
}

/* All intersecting pairs, sorted by (a, b); writes up to `capacity`, returns the total (-1: OOM). */
int64_t oracle_polygon_join(const int32_t* xy1, const int64_t* ro1, const int64_t* pro1, int32_t n1,
                            const int32_t* xy2, const int64_t* ro2, const int64_t* pro2, int32_t n2,
                            int32_t* out_a, int32_t* out_b, int64_t capacity, int nthreads) {
    if (n1 <= 0 || n2 <= 0) return 0;
    uint8_t* hit = (uint8_t*)calloc((size_t)n1 * (size_t)n2, 1);
    if (nthreads < 1) nthreads = 1;
    if (nthreads > n1) nthreads = n1;
    pj_task* tasks = (pj_task*)calloc(nthreads, sizeof(pj_task));
    pthread_t* th = (pthread_t*)calloc(nthreads, sizeof(pthread_t));
    if (!hit || !tasks || !th) { free(hit); free(tasks); free(th); return -1; }
    for (int t = 0; t < nthreads; ++t) {
        pj_task* k = &tasks[t];
        k->A = (pset){xy1, ro1, pro1, n1};
        k->B = (pset){xy2, ro2, pro2, n2};
        k->a0 = (int32_t)((int64_t)n1 * t / nthreads);
        k->a1 = (int32_t)((int64_t)n1 * (t + 1) / nthreads);
        k->hit = hit;
        pthread_create(&th[t], NULL, pj_worker, k);
    }
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    int64_t total = 0;
    for (int32_t a = 0; a < n1; ++a)
        for (int32_t b = 0; b < n2; ++b)
            if (hit[(int64_t)a * n2 + b]) {
                if (total < capacity) { out_a[total] = a; out_b[total] = b; }
                ++total;
            }
    free(hit); free(tasks); free(th);
    return total;
}
