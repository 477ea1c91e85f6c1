/*
 * rtree_join.c — a simple CPU R-tree join, the second CPU baseline named by BASELINE.json's
 * north_star ("reported next to the oracle (and a simple R-tree CPU join)").  TEST / BASELINE
 * INFRASTRUCTURE ONLY, like the oracle: nothing on the CUDA path uses it.
 *
 * Filter: an STR (sort-tile-recursive) bulk-loaded R-tree over polygon bounding boxes, fanout
 * 16; refine: the same half-open even-odd predicate as the oracle (reading C1), over
 * every ring of each candidate polygon.  Parallel over points with pthreads.  Results are
 * identical to the oracle's (checked in tests/test_oracle_pins.py).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

#define RT_FAN 16

typedef struct { int64_t x0, y0, x1, y1; int32_t child; int32_t count; } rt_node;  /* child<0: leaf run of polygons */

typedef struct {
    rt_node* nodes; int32_t nn, cap, root;
    int32_t* leaf_poly;         /* polygon ids in STR order */
    int64_t (*bb)[4];
} rtree;

static int rt_edge(int64_t ax, int64_t ay, int64_t bx, int64_t by, int64_t px, int64_t py) {
    if ((ay > py) == (by > py)) return 0;
    __int128 o = (__int128)(bx - ax) * (py - ay) - (__int128)(by - ay) * (px - ax);
    return by > ay ? (o > 0) : (o < 0);
}

static int rt_inside(const int32_t* xy, const int64_t* ro, int64_t r0, int64_t r1, int64_t px, int64_t py) {
    int par = 0;
    for (int64_t r = r0; r < r1; ++r)
        for (int64_t k = ro[r]; k < ro[r + 1]; ++k) {
            int64_t k2 = k + 1 < ro[r + 1] ? k + 1 : ro[r];
            par ^= rt_edge(xy[2 * k], xy[2 * k + 1], xy[2 * k2], xy[2 * k2 + 1], px, py);
        }
    return par;
}

static int64_t (*g_bb)[4];
static int cmp_cx(const void* a, const void* b) {
    int64_t u = g_bb[*(const int32_t*)a][0] + g_bb[*(const int32_t*)a][2];
    int64_t v = g_bb[*(const int32_t*)b][0] + g_bb[*(const int32_t*)b][2];
    return (u > v) - (u < v);
}
static int cmp_cy(const void* a, const void* b) {
    int64_t u = g_bb[*(const int32_t*)a][1] + g_bb[*(const int32_t*)a][3];
    int64_t v = g_bb[*(const int32_t*)b][1] + g_bb[*(const int32_t*)b][3];
    return (u > v) - (u < v);
}

static int32_t rt_add(rtree* t, rt_node nd) {
    if (t->nn == t->cap) { t->cap = t->cap ? 2 * t->cap : 64; t->nodes = (rt_node*)realloc(t->nodes, sizeof(rt_node) * t->cap); }
    t->nodes[t->nn] = nd;
    return t->nn++;
}

/* builds one level: groups of RT_FAN consecutive items -> parent nodes; returns first parent */
static void rt_build(rtree* t, int32_t P) {
    int32_t* ids = (int32_t*)malloc(sizeof(int32_t) * (P > 0 ? P : 1));
    for (int32_t i = 0; i < P; ++i) ids[i] = i;
    g_bb = t->bb;
    /* STR leaf packing: sort by x centre, cut into sqrt(#leaves) slices, sort each by y centre */
    int32_t nleaf = (P + RT_FAN - 1) / RT_FAN, slices = 1;
    while ((int64_t)slices * slices < nleaf) ++slices;
    qsort(ids, P, sizeof(int32_t), cmp_cx);
    int32_t per_slice = slices * RT_FAN;
    for (int32_t s0 = 0; s0 < P; s0 += per_slice) {
        int32_t n = P - s0 < per_slice ? P - s0 : per_slice;
        qsort(ids + s0, n, sizeof(int32_t), cmp_cy);
    }
    t->leaf_poly = ids;
    int32_t lvl0 = t->nn;
    for (int32_t i = 0; i < P; i += RT_FAN) {
        rt_node nd = {INT64_MAX, INT64_MAX, INT64_MIN, INT64_MIN, -1 - i, P - i < RT_FAN ? P - i : RT_FAN};
        for (int32_t k = i; k < i + nd.count; ++k) {
            int64_t* b = t->bb[ids[k]];
            if (b[0] < nd.x0) nd.x0 = b[0]; if (b[1] < nd.y0) nd.y0 = b[1];
            if (b[2] > nd.x1) nd.x1 = b[2]; if (b[3] > nd.y1) nd.y1 = b[3];
        }
        rt_add(t, nd);
    }
    int32_t lo = lvl0, hi = t->nn;
    while (hi - lo > 1) {
        for (int32_t i = lo; i < hi; i += RT_FAN) {
            rt_node nd = {INT64_MAX, INT64_MAX, INT64_MIN, INT64_MIN, i, hi - i < RT_FAN ? hi - i : RT_FAN};
            for (int32_t k = i; k < i + nd.count; ++k) {
                rt_node* c = &t->nodes[k];
                if (c->x0 < nd.x0) nd.x0 = c->x0; if (c->y0 < nd.y0) nd.y0 = c->y0;
                if (c->x1 > nd.x1) nd.x1 = c->x1; if (c->y1 > nd.y1) nd.y1 = c->y1;
            }
            rt_add(t, nd);
        }
        lo = hi; hi = t->nn;
    }
    t->root = hi - 1;
}

typedef struct {
    const rtree* t; const int32_t* pts; int64_t i0, i1;
    const int32_t* xy; const int64_t* ro; const int64_t* pro; int64_t* counts; int32_t P;
} rt_task;

static void* rt_worker(void* arg) {
    rt_task* k = (rt_task*)arg;
    const rtree* t = k->t;
    int32_t stack[256];
    for (int64_t i = k->i0; i < k->i1; ++i) {
        int64_t px = k->pts[2 * i], py = k->pts[2 * i + 1];
        int sp = 0;
        if (t->nn > 0) stack[sp++] = t->root;
        while (sp > 0) {
            const rt_node* nd = &t->nodes[stack[--sp]];
            if (px < nd->x0 || px > nd->x1 || py < nd->y0 || py > nd->y1) continue;
            if (nd->child < 0) {
                int32_t s = -1 - nd->child;
                for (int32_t q = s; q < s + nd->count; ++q) {
                    int32_t p = t->leaf_poly[q];
                    const int64_t* b = t->bb[p];
                    if (px < b[0] || px > b[2] || py < b[1] || py > b[3]) continue;
                    if (rt_inside(k->xy, k->ro, k->pro[p], k->pro[p + 1], px, py)) k->counts[p]++;
                }
            } else {
                for (int32_t c = nd->child; c < nd->child + nd->count && sp < 256; ++c) stack[sp++] = c;
            }
        }
    }
    return NULL;
}

/* COUNT via the R-tree; counts[P] overwritten.  Returns 0, or -1 on allocation failure. */
int rtree_join_count(const int32_t* pts, int64_t n, const int32_t* xy, const int64_t* ro, const int64_t* pro,
                     int32_t P, int64_t* counts, int nthreads) {
    rtree t;
    memset(&t, 0, sizeof(t));
    t.bb = (int64_t(*)[4])malloc(sizeof(int64_t) * 4 * (P > 0 ? P : 1));
    if (!t.bb) return -1;
    for (int32_t p = 0; p < P; ++p) {
        int64_t* b = t.bb[p];
        b[0] = b[1] = INT64_MAX; b[2] = b[3] = INT64_MIN;
        for (int64_t r = pro[p]; r < pro[p + 1]; ++r)
            for (int64_t k = ro[r]; k < ro[r + 1]; ++k) {
                int64_t x = xy[2 * k], y = xy[2 * k + 1];
                if (x < b[0]) b[0] = x; if (y < b[1]) b[1] = y;
                if (x > b[2]) b[2] = x; if (y > b[3]) b[3] = y;
            }
    }
    rt_build(&t, P);
    if (nthreads < 1) nthreads = 1;
    rt_task* tasks = (rt_task*)calloc(nthreads, sizeof(rt_task));
    pthread_t* th = (pthread_t*)calloc(nthreads, sizeof(pthread_t));
    memset(counts, 0, sizeof(int64_t) * (size_t)P);
    for (int i = 0; i < nthreads; ++i) {
        rt_task* k = &tasks[i];
        k->t = &t; k->pts = pts; k->i0 = n * i / nthreads; k->i1 = n * (i + 1) / nthreads;
        k->xy = xy; k->ro = ro; k->pro = pro; k->P = P;
        k->counts = (int64_t*)calloc(P > 0 ? P : 1, sizeof(int64_t));
        pthread_create(&th[i], NULL, rt_worker, k);
    }
    for (int i = 0; i < nthreads; ++i) {
        pthread_join(th[i], NULL);
        for (int32_t p = 0; p < P; ++p) counts[p] += tasks[i].counts[p];
        free(tasks[i].counts);
    }
    free(tasks); free(th); free(t.nodes); free(t.leaf_poly); free(t.bb);
    return 0;
}
