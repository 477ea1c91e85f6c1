/*
 * distance_oracle.c — CPU ORACLE for SPADE's distance-based queries over points and its kNN
 * selection (TEST INFRASTRUCTURE ONLY; same rules as spade_oracle.c: only tests/, smoke() and
 * bench.py's CPU legs load it; it shares no code with the CUDA path).
 *
 * What it computes (brute force over EVERY (point, disk) pair):
 *
 *   within(i, d) = (px - cx_d)^2 + (py - cy_d)^2 <= r2_d            (exact, __int128)
 *
 *   counts[d] = |{ i : within(i, d) }|                                    (int64)
 *   pairs     = { (point_id_base + i, d) : within(i, d) }  sorted by (point, disk)
 *   select    = { point_id_base + i : exists d with within(i, d) }        ascending
 *   knn(q, k) = the k points smallest in (dist2(i, q), point id)          in that order
 *
 * r2_d is the SQUARED radius as an integer: for integer points, distance <= r  <=>
 * dist2 <= floor(r^2), so any real radius is represented exactly (reading D2).
 *
 * Passages followed (PAPER.md line numbers):
 *   - distance constraint w.r.t. a point = a circle of radius r (interior AND boundary)
 *   - distance-based selections / joins differ from spatial ones only in the canvas
 *   - type 1 join: pairs with distance(x_i, y_j) <= r (one r)
 *   - type 2 join: pairs with distance(x_i, y_j) <= r_i (one r per object of D1)
 *   - kNN selection: the k points closest to a query point p
 *     (the paper's 3-step circle plan P:218-228 is HOW the GPU path finds them; the oracle
 *      is the definition: sort every point by distance and keep the first k)
 * Readings: D1 closed disk (<=); D2 squared integer radii; D3 ties in kNN broken by
 * point id (a total order, so the answer is unique); D4 a point joins every disk containing it.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

/* One (point, disk) pair: is the point within distance sqrt(r2) of the centre? */
int oracle_in_disk(int64_t px, int64_t py, int64_t cx, int64_t cy, int64_t r2) {
    __int128 dx = (__int128)px - cx, dy = (__int128)py - cy;
    return dx * dx + dy * dy <= (__int128)r2;
}

typedef struct {
    const int32_t* xy; int64_t i0, i1;
    const int32_t* cxy; const int64_t* r2; int32_t nd;
    int64_t* counts;
    int64_t* pt; int32_t* pl; int64_t n_pairs, cap_pairs; int oom;
    int want_pairs;
} disk_task;

static void* disk_worker(void* arg) {
    disk_task* t = (disk_task*)arg;
    for (int64_t i = t->i0; i < t->i1; ++i) {
        int64_t px = t->xy[2 * i], py = t->xy[2 * i + 1];
        for (int32_t d = 0; d < t->nd; ++d) {
            if (!oracle_in_disk(px, py, t->cxy[2 * d], t->cxy[2 * d + 1], t->r2[d])) continue;
            if (t->counts) t->counts[d] += 1;
            if (t->want_pairs) {
                if (t->n_pairs == t->cap_pairs) {
                    int64_t nc = t->cap_pairs ? 2 * t->cap_pairs : 1024;
                    int64_t* npt = (int64_t*)realloc(t->pt, nc * sizeof(int64_t));
                    int32_t* npl = (int32_t*)realloc(t->pl, nc * sizeof(int32_t));
                    if (!npt || !npl) { t->oom = 1; if (npt) t->pt = npt; if (npl) t->pl = npl; return NULL; }
                    t->pt = npt; t->pl = npl; t->cap_pairs = nc;
                }
                t->pt[t->n_pairs] = i; t->pl[t->n_pairs] = d; t->n_pairs++;
            }
        }
    }
    return NULL;
}

/* Brute force over all pairs, threads over contiguous point ranges.  counts (if given) are
 * overwritten; pairs are written in (point, disk) order up to capacity; returns the total. */
static int64_t disk_run(const int32_t* xy, int64_t n, const int32_t* cxy, const int64_t* r2, int32_t nd,
                        int nthreads, int64_t* counts, int want_pairs, int64_t point_id_base,
                        int64_t* out_pt, int32_t* out_pl, int64_t capacity) {
    if (nthreads < 1) nthreads = 1;
    if (n < nthreads) nthreads = n > 0 ? (int)n : 1;
    disk_task* tasks = (disk_task*)calloc(nthreads, sizeof(disk_task));
    pthread_t* th = (pthread_t*)calloc(nthreads, sizeof(pthread_t));
    if (!tasks || !th) { free(tasks); free(th); return -1; }
    for (int t = 0; t < nthreads; ++t) {
        disk_task* k = &tasks[t];
        k->xy = xy; k->i0 = n * t / nthreads; k->i1 = n * (t + 1) / nthreads;
        k->cxy = cxy; k->r2 = r2; k->nd = nd; k->want_pairs = want_pairs;
        k->counts = counts ? (int64_t*)calloc(nd > 0 ? nd : 1, sizeof(int64_t)) : NULL;
        pthread_create(&th[t], NULL, disk_worker, k);
    }
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    if (counts) memset(counts, 0, sizeof(int64_t) * (size_t)nd);
    int64_t total = 0; int failed = 0;
    for (int t = 0; t < nthreads; ++t) {
        disk_task* k = &tasks[t];
        if (k->oom) failed = 1;
        if (counts) for (int32_t d = 0; d < nd; ++d) counts[d] += k->counts[d];
        for (int64_t q = 0; q < k->n_pairs; ++q, ++total) {
            if (total < capacity) {
                if (out_pt) out_pt[total] = point_id_base + k->pt[q];
                if (out_pl) out_pl[total] = k->pl[q];
            }
        }
        free(k->counts); free(k->pt); free(k->pl);
    }
    free(tasks); free(th);
    return failed ? -1 : total;
}

/* Per-disk COUNT (the aggregation of P:214 over distance canvases). */
int oracle_disk_join_count(const int32_t* xy, int64_t n, const int32_t* cxy, const int64_t* r2, int32_t nd,
                           int64_t* counts, int nthreads) {
    return disk_run(xy, n, cxy, r2, nd, nthreads, counts, 0, 0, NULL, NULL, 0) < 0 ? -1 : 0;
}

/* Distance join pairs (P:208 type 1 / P:210 type 2), sorted by (point, disk). */
int64_t oracle_disk_join_pairs(const int32_t* xy, int64_t n, int64_t point_id_base, const int32_t* cxy,
                               const int64_t* r2, int32_t nd, int64_t* out_pt, int32_t* out_pl, int64_t capacity,
                               int nthreads) {
    return disk_run(xy, n, cxy, r2, nd, nthreads, NULL, 1, point_id_base, out_pt, out_pl, capacity);
}

/* Distance selection (P:204 with P:184): ids of points within at least one disk, ascending. */
int64_t oracle_disk_select(const int32_t* xy, int64_t n, int64_t point_id_base, const int32_t* cxy,
                           const int64_t* r2, int32_t nd, int64_t* out_ids, int64_t capacity, int nthreads) {
    int64_t np = disk_run(xy, n, cxy, r2, nd, nthreads, NULL, 1, 0, NULL, NULL, 0);
    if (np < 0) return -1;
    int64_t* pt = (int64_t*)malloc(sizeof(int64_t) * (size_t)(np > 0 ? np : 1));
    if (!pt) return -1;
    disk_run(xy, n, cxy, r2, nd, nthreads, NULL, 1, 0, pt, NULL, np);
    int64_t total = 0;
    for (int64_t q = 0; q < np; ++q) {
        if (q > 0 && pt[q] == pt[q - 1]) continue;         /* pairs are grouped by point */
        if (total < capacity) out_ids[total] = point_id_base + pt[q];
        total++;
    }
    free(pt);
    return total;
}

/* kNN selection: the k points nearest to (qx, qy), ties by point id.  Plain definition:
 * every point's squared distance, one sort of all n (dist2, id) keys, the first min(k, n). */
typedef struct { __int128 d2; int64_t id; } knn_key;

static int knn_cmp(const void* a, const void* b) {
    const knn_key* x = (const knn_key*)a; const knn_key* y = (const knn_key*)b;
    if (x->d2 != y->d2) return x->d2 < y->d2 ? -1 : 1;
    return (x->id > y->id) - (x->id < y->id);
}

int64_t oracle_knn(const int32_t* xy, int64_t n, int64_t point_id_base, int64_t qx, int64_t qy, int64_t k,
                   int64_t* out_ids, int64_t* out_d2) {
    if (k > n) k = n;
    if (k <= 0) return 0;
    knn_key* a = (knn_key*)malloc(sizeof(knn_key) * (size_t)n);
    if (!a) return -1;
    for (int64_t i = 0; i < n; ++i) {
        __int128 dx = (__int128)xy[2 * i] - qx, dy = (__int128)xy[2 * i + 1] - qy;
        a[i].d2 = dx * dx + dy * dy;
        a[i].id = point_id_base + i;
    }
    qsort(a, (size_t)n, sizeof(knn_key), knn_cmp);
    for (int64_t i = 0; i < k; ++i) {
        out_ids[i] = a[i].id;
        if (out_d2) out_d2[i] = (int64_t)a[i].d2;
    }
    free(a);
    return k;
}
