/*
 * spade.h — C ABI of the B200-native SPADE point-in-polygon join (paper_conf_icde_doraiswamyf22_b200).
 *
 * The method (Doraiswamy & Freire, "GPU-Powered Spatial Database Engine for Commodity Hardware",
 * ICDE'22; citations are /root/reference/PAPER.md line numbers "P:n"):
 *   polygons are rasterised into a DISCRETE CANVAS whose pixels hold either the owning polygon or a
 *   pointer into a BOUNDARY INDEX (Sec. 4.1; Sec. 4.3); points are looked up in
 *   that canvas and only points on boundary pixels get an exact test (Sec. 5.1-5.2).
 *   Here the boundary index maps a run of boundary pixels to the exact list of edges touching it
 *   plus the polygon set just right of the run, so results are EXACT.
 *
 * Results are defined by the half-open even-odd rule (reading C1): point (px,py) is in
 * polygon p iff the number of edges (a,b) over all rings of p with (a.y>py) != (b.y>py) whose
 * crossing with the line y=py lies strictly right of px is odd.  All arithmetic is exact integer.
 *
 * Conventions for every entry point:
 *   - array arguments are DEVICE pointers (cudaMalloc / torch CUDA tensors) unless the name ends
 *     in _host; all work is enqueued on `stream` (a cudaStream_t, e.g. torch's current stream);
 *   - coordinates are int32 fixed point; points are int32 (x, y) pairs interleaved, N x 8 bytes,
 *     any 8-byte alignment (32-byte alignment is fastest);
 *   - point ids are int64: point_id_base + index of the point in the call's array;
 *   - polygon ids are the index 0..P-1 of the polygon in the canvas's input;
 *   - the return value is a status code (SPADE_OK or a negative SPADE_ERR_*); nothing throws
 *     across the ABI; spade_last_error() gives a thread-local detail message;
 *   - no host<->device synchronisation unless stated.
 * The library owns the canvas and its device memory; the caller owns every other buffer.
 */
#ifndef SPADE_H
#define SPADE_H

#include <stdint.h>

#if defined(__GNUC__)
#define SPADE_API __attribute__((visibility("default")))
#else
#define SPADE_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct spade_canvas spade_canvas;   /* opaque; owns its device memory */
typedef struct CUstream_st* spade_stream_t;  /* == cudaStream_t (NULL = legacy default stream) */

enum {
    SPADE_OK = 0,
    SPADE_ERR_INVALID_ARG = -1,  /* null pointer, negative size, malformed offsets        */
    SPADE_ERR_COORD_RANGE = -2,  /* a polygon vertex outside [-2^30, 2^30)                 */
    SPADE_ERR_CAPACITY = -3,     /* output capacity too small; *n_out = required count     */
    SPADE_ERR_CUDA = -4,         /* a CUDA runtime error (detail in spade_last_error)      */
    SPADE_ERR_OOM = -5,          /* device or host allocation failed                       */
    SPADE_ERR_INTERNAL = -6      /* an internal consistency check failed (a bug)           */
};

/* Canvas resolution (reading C5; the paper fixes no resolution for constraint
 * canvases).  Pixel = 2^log2_pixel grid units.  log2_pixel = -1 selects the smallest s with
 * max(W, H) <= max_dim, where W = ((maxx-minx) >> s) + 1 over the polygon extent.  Results do
 * not depend on the resolution; only speed and memory do. */
typedef struct {
    int32_t log2_pixel;   /* -1 = auto                                    */
    int32_t max_dim;      /* used when log2_pixel == -1; 0 means 4096     */
    int32_t flags;        /* SPADE_CANVAS_* bits; 0 = defaults            */
} spade_canvas_params;

/* flags: keep the dense W x H fine canvas as the probe's second level even when the compact
 * mixed-tile layout applies (for tests / comparisons; results are identical). */
#define SPADE_CANVAS_DENSE 1
/* flags: no 16-bit copy of a dense second level (the probe then gathers the int32 canvas).  By
 * default a dense second level over fewer than 65534 polygons is probed through a uint16 copy
 * (owner id / empty / "record": half the gather footprint; records are looked up in the int32
 * canvas by the exact-test stage).  Results are identical either way. */
#define SPADE_CANVAS_NO_FINE16 2

/* Build the discrete canvas + boundary index for a polygon set (P:113-123 canvas creation,
 * Sec. 4.2; P:146 and P:268 boundary index, Sec. 4.3 / 5.5).
 *   ring_xy       [V*2]  int32 vertex coordinates (x,y) of all rings, each ring implicitly closed
 *                        (last vertex connects to first); every coordinate in [-2^30, 2^30)
 *   ring_off      [R+1]  int64: ring r = vertices [ring_off[r], ring_off[r+1]); ring_off[0] = 0
 *   poly_ring_off [P+1]  int64: polygon p = rings [poly_ring_off[p], poly_ring_off[p+1]);
 *                        poly_ring_off[0] = 0, poly_ring_off[P] = R.  Polygons may have holes,
 *                        several outer rings, self-intersections and degenerate rings
 *                        (even-odd over all rings, reading C2); polygons may overlap (C3).
 *   num_polys     P >= 0
 *   prm           NULL = defaults {-1, 4096, 0}
 *   out           receives the canvas handle (NULL on error)
 * The input buffers may be freed once this returns.  Synchronises `stream` (a few times: sizes
 * are data dependent).  Errors: INVALID_ARG, COORD_RANGE, OOM, CUDA. */
SPADE_API int spade_build_canvas(const int32_t* ring_xy, const int64_t* ring_off, const int64_t* poly_ring_off,
                       int32_t num_polys, const spade_canvas_params* prm, spade_stream_t stream,
                       spade_canvas** out);

/* Build a DISTANCE canvas ("Canvases for Distance-Based Queries", Sec. 4.2; used by the
 * distance-based selections and joins of P:204-210, Sec. 5.2): one closed disk per constraint,
 *   disk d = { (x, y) : (x - cx_d)^2 + (y - cy_d)^2 <= r2_d }      (readings D1-D4)
 * The squared radius is an integer: for integer points "distance <= r" is exactly
 * "dist2 <= floor(r^2)", so any real radius r is represented by r2 = floor(r^2).
 *   center_xy [D*2] int32 disk centres (x, y) interleaved
 *   r2        [D]   int64 squared radii, 0 <= r2 < 2^62
 *   num_disks D >= 0; the disk id of center_xy[d] is d
 * Type 1 distance join (one r): all r2 equal.  Type 2 (per-object r_i): per-disk r2.
 * Every disk's integer points must lie in [-2^30, 2^30)^2: cx - isqrt(r2) >= -2^30 and
 * cx + isqrt(r2) < 2^30 (same for y), else SPADE_ERR_COORD_RANGE; r2 out of range or NULL
 * arrays: SPADE_ERR_INVALID_ARG.  The canvas is used with the same calls as a polygon canvas
 * (spade_join_count, spade_select, spade_join_pairs, spade_join_count_host), with "polygon id"
 * meaning disk id and "inside" meaning within the closed disk; disks may overlap (a point joins
 * every disk containing it).  Ownership and synchronisation as spade_build_canvas. */
SPADE_API int spade_build_disk_canvas(const int32_t* center_xy, const int64_t* r2, int32_t num_disks,
                            const spade_canvas_params* prm, spade_stream_t stream, spade_canvas** out);

/* Release a canvas (NULL is a no-op).  Synchronises the canvas's device.  Every call taking a
 * canvas runs on the device the canvas was built on (made current for the call and restored). */
SPADE_API void spade_canvas_free(spade_canvas* c);

/* Canvas statistics for reports: fine canvas W x H at 2^log2_pixel units per pixel; coarse
 * (shared-memory) tile grid Wc x Hc of 2^log2_tile fine pixels per side; number of boundary
 * runs (+ multi-owner records) and of listed run edges; fraction of coarse tiles that are mixed.
 * Any output pointer may be NULL. */
SPADE_API int spade_canvas_info(const spade_canvas* c, int32_t* W, int32_t* H, int32_t* log2_pixel,
                      int32_t* Wc, int32_t* Hc, int32_t* log2_tile,
                      int64_t* num_runs, int64_t* num_run_edges, double* mixed_tile_frac);

/* Build profile (the paper's "polygon processing" cost): device time of each stage of
 * this canvas's build, from CUDA events recorded on the build stream at the stage boundaries
 * (each stage is also an NVTX range "spade_build:<name>").  Writes min(cap, stages) values (ms)
 * and returns the number of stages (< 0: error); spade_canvas_build_stage_name(i) names stage i
 * (NULL past the last).  Stages: K-B0 edges + extent, K-B1 fragments + events, K-B2 boundary
 * pixels + pixel-local edge lists, K-B3 corner owner sets, K-B4/B6 K sets + packed records,
 * K-B5 coarse tiles + compact / 16-bit levels.  An empty canvas has 0 stages. */
SPADE_API int spade_canvas_build_times(const spade_canvas* c, float* ms, int32_t cap);
SPADE_API const char* spade_canvas_build_stage_name(int32_t i);

/* 64-bit checksum of everything the probe reads from the canvas (geometry, fine / compact /
 * coarse levels, records, primitive blobs, owner sets), written to *out (HOST).  Equal polygon
 * arrays give equal checksums on any device (the build is deterministic); ranks that replicate a
 * canvas compare them (multi-GPU is the paper's future work).
 * Synchronises `stream`.  Errors: INVALID_ARG (NULL), CUDA, OOM. */
SPADE_API int spade_canvas_checksum(const spade_canvas* c, uint64_t* out, spade_stream_t stream);

/* Aggregation: per-polygon COUNT of the points of xy[0..n) inside each polygon (P:214,
 * Sec. 5.2, "aggregation plan 2" for points: partial aggregates without materialising the join).
 *   xy      [n*2] int32 device points
 *   counts  [P]   int64 device counts, ACCUMULATED INTO (the caller zeroes them)
 * Asynchronous (no host sync).  n == 0 is a no-op.  Errors: INVALID_ARG, CUDA. */
SPADE_API int spade_join_count(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t* counts,
                     spade_stream_t stream);

/* Selection (Sec. 5.2): ids of the points inside AT LEAST ONE polygon of the canvas
 * (a 1-polygon canvas is the paper's polygonal selection), each id once, order unspecified.
 *   out_ids   [capacity] int64 device
 *   n_out     HOST int64: number of selected points
 * Map with n_max = n is the paper's 1-pass Map: capacity >= n always suffices.
 * If capacity < needed: returns SPADE_ERR_CAPACITY with *n_out = needed, out_ids unspecified;
 * call again with a larger buffer (the paper's 2-pass Map).  Synchronises `stream`. */
SPADE_API int spade_select(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t point_id_base,
                 int64_t* out_ids, int64_t capacity, int64_t* n_out, spade_stream_t stream);

/* Join (pair form P:208): all (point_id, polygon_id) with the point inside the
 * polygon, as two device arrays (SoA), order unspecified.  n_max = n when polygons do not
 * overlap.  Capacity protocol and synchronisation as spade_select. */
SPADE_API int spade_join_pairs(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t point_id_base,
                     int64_t* out_point_ids, int32_t* out_poly_ids, int64_t capacity,
                     int64_t* n_out, spade_stream_t stream);

/* End-to-end COUNT from HOST memory: streams xy_host[0..n) to the device in chunks (copies
 * overlapped with the probe on two internal streams; pinned memory gives full PCIe bandwidth),
 * and ACCUMULATES the int64 counts into counts_host[P].  Synchronises `stream` before return.
 * This is the user-facing call for point sets that live on the host (the
 * paper's times are dominated by exactly this host->GPU transfer). */
SPADE_API int spade_join_count_host(const spade_canvas* c, const int32_t* xy_host, int64_t n,
                          int64_t* counts_host, spade_stream_t stream);

/* Host-resident SELECT / PAIRS (out-of-core point streams, Sec. 5.3; the
 * I/O-GPU pipelining of P:480): as spade_select / spade_join_pairs, but xy_host and the outputs
 * are HOST arrays (pinned memory gives full PCIe bandwidth; pageable works, slower).  The points
 * are streamed in chunks (spade_set_option "host_chunk", default 2^25 points): the H2D copy of
 * chunk k+1, the probe of chunk k and the D2H copy of chunk k-1's results run on three internal
 * streams.  Results come in chunk order, unspecified order within a chunk.  Capacity protocol as
 * spade_select: `capacity` < total -> SPADE_ERR_CAPACITY with *n_out = total (the first
 * `capacity` results are written); n_max = n for select and for pairs over
 * non-overlapping polygons.  Device memory used: 2 staging + 2 result buffers of one
 * chunk each (a chunk whose PAIRS exceed one chunk is re-run with a larger buffer).
 * Synchronises `stream` before return.  Errors: INVALID_ARG, CAPACITY, CUDA, OOM. */
SPADE_API int spade_select_host(const spade_canvas* c, const int32_t* xy_host, int64_t n, int64_t point_id_base,
                                int64_t* out_ids_host, int64_t capacity, int64_t* n_out, spade_stream_t stream);
SPADE_API int spade_join_pairs_host(const spade_canvas* c, const int32_t* xy_host, int64_t n,
                                    int64_t point_id_base, int64_t* out_point_ids_host,
                                    int32_t* out_poly_ids_host, int64_t capacity, int64_t* n_out,
                                    spade_stream_t stream);

/* Polygon x Polygon join (Sec. 5.2): all pairs (a, b), polygon a of D1 and polygon b of D2,
 * whose CLOSED regions intersect (ST_INTERSECTS; touching boundaries count; DESIGN.md
 * reading C15), sorted by (a, b), each pair once.  Both sets use spade_build_canvas's layout
 * (device arrays; even-odd regions over all rings of a polygon) and must be VALID polygons:
 * rings of >= 3 vertices, no zero-length edge, no segment used twice by one polygon (rings may
 * touch at points; different polygons may share edges).  `prm` (may be NULL) sets the resolution
 * of the common pixel grid both sets are rasterised on (max_dim over the union extent, or
 * log2_pixel); results do not depend on it.  The join tests the local edge pairs of pixels that
 * are boundary pixels of both canvases (exact closed-segment test) and probes every ring's first
 * vertex against the other set's canvas (the point join).
 *   out_a, out_b [capacity] int32 device (polygon ids in D1, D2);  n_out HOST: number of pairs.
 * capacity < n_out -> SPADE_ERR_CAPACITY (the first `capacity` pairs in order are written).
 * Vertices outside [-2^30, 2^30) -> SPADE_ERR_COORD_RANGE.  Synchronises `stream`. */
SPADE_API int spade_join_polygons(const int32_t* ring_xy1, const int64_t* ring_off1, const int64_t* poly_ring_off1,
                                  int32_t num_polys1, const int32_t* ring_xy2, const int64_t* ring_off2,
                                  const int64_t* poly_ring_off2, int32_t num_polys2, const spade_canvas_params* prm,
                                  int32_t* out_a, int32_t* out_b, int64_t capacity, int64_t* n_out, spade_stream_t stream);

/* ---- Layer index ---------------------------------------------------
 * The paper's plan for overlapping polygon sets: layers of mutually non-intersecting polygons, one
 * canvas and one pass over the points per layer.  (spade_build_canvas handles overlaps exactly in
 * ONE canvas with owner sets; this is the alternative plan, kept for comparison: DESIGN.md §6.)
 *
 * spade_layer_assign: greedy colouring (Welsh-Powell) of the conflict graph given as npairs HOST
 *   pairs (pair_a[i], pair_b[i]) of polygon ids in [0, P) (self pairs and duplicates allowed):
 *   layer_of [P] HOST output, layer of each polygon, such that no pair shares a layer;
 *   num_layers HOST output.  Host-only (no device work).  Ids out of range -> INVALID_ARG.
 * spade_build_layered: conflicts = the closed-intersection self-join of the set
 *   (spade_join_polygons; touching polygons conflict too), layers by spade_layer_assign, then one
 *   spade_build_canvas per layer over all P polygon slots (the other layers' polygons get no
 *   rings), so every layer's COUNT uses global polygon ids.  Arguments as spade_build_canvas (device
 *   arrays, which must be VALID polygons as for spade_join_polygons); `*out` owns the canvases
 *   (spade_layered_free).  Synchronises `stream`.
 * spade_join_count_layered: COUNT as spade_join_count, one probe pass per layer, ACCUMULATED into
 *   the device counts [P] (the caller zeroes them).
 * spade_layered_info: number of layers; layer_of [P] HOST (may be NULL).
 * spade_layered_free: frees the layers (NULL: no-op). */
typedef struct spade_layered spade_layered;
SPADE_API int spade_layer_assign(const int32_t* pair_a, const int32_t* pair_b, int64_t npairs, int32_t num_polys,
                                 int32_t* layer_of, int32_t* num_layers);
SPADE_API int spade_build_layered(const int32_t* ring_xy, const int64_t* ring_off, const int64_t* poly_ring_off,
                                  int32_t num_polys, const spade_canvas_params* prm, spade_stream_t stream,
                                  spade_layered** out);
SPADE_API int spade_join_count_layered(const spade_layered* layered, const int32_t* xy, int64_t n, int64_t* counts,
                                       spade_stream_t stream);
SPADE_API int spade_layered_info(const spade_layered* layered, int32_t* num_layers, int32_t* layer_of);
SPADE_API void spade_layered_free(spade_layered* layered);

/* ---- kNN selection over points (Sec. 5.2), in the paper's three steps ------------
 * The circles of step 1 are concentric around the query q with squared radii
 *   r2_b = the largest squared distance of bucket b,  b = 0 .. SPADE_KNN_BINS-1, where
 *   bucket(d2) = d2 (d2 < 4),  4 + 4(e-2) + ((d2 >> (e-2)) & 3) (d2 >= 4, e = floor(log2 d2))
 * (consecutive radii differ by a factor <= sqrt(1.25): the paper's r_i = r_max / alpha^i with
 * the circles aligned to quarter-octaves of the squared distance).
 * Coordinates of the query and of every point must lie in [-2^30, 2^30) (squared distances are
 * then exact in int64); points outside are counted in hist[SPADE_KNN_BINS] and make spade_knn
 * fail with SPADE_ERR_COORD_RANGE.  The result is unique: the k points smallest in
 * (squared distance, point id) (reading D3). */
#define SPADE_KNN_BINS 248

/* Step 1: aggregation over the circles.  ACCUMULATES into hist[SPADE_KNN_BINS + 1]
 * (int64, device): hist[b] = points in bucket b, hist[SPADE_KNN_BINS] = out-of-range points;
 * COUNT(circle b) = hist[0] + ... + hist[b].  Asynchronous.  Sum the histograms of several point
 * shards (e.g. all_reduce) before step 2. */
SPADE_API int spade_knn_histogram(const int32_t* xy, int64_t n, int32_t qx, int32_t qy, int64_t* hist,
                        spade_stream_t stream);

/* Between steps 1 and 2 (host): the smallest circle b with COUNT(circle b) >= k (the last
 * circle if fewer than k points exist).  hist_host[SPADE_KNN_BINS + 1] as above.  Outputs its
 * squared radius and its count (the number of candidates step 2 returns). */
SPADE_API int spade_knn_radius(const int64_t* hist_host, int64_t k, int64_t* r2_out, int64_t* count_out);

/* Step 2: distance selection — ids (point_id_base + index) and squared distances of the
 * points with dist2 <= r2, order unspecified, capacity protocol of spade_select.  Syncs. */
SPADE_API int spade_knn_select(const int32_t* xy, int64_t n, int64_t point_id_base, int32_t qx, int32_t qy,
                     int64_t r2, int64_t* out_ids, int64_t* out_d2, int64_t capacity, int64_t* n_out,
                     spade_stream_t stream);

/* Step 3: sort m candidates (ids >= 0, d2 as from step 2) by (d2, id) and write the
 * first min(k, m) to out_ids / out_d2 (out_d2 may be NULL).  Asynchronous. */
SPADE_API int spade_knn_topk(const int64_t* ids, const int64_t* d2, int64_t m, int64_t k, int64_t* out_ids,
                   int64_t* out_d2, spade_stream_t stream);

/* All three steps on one device: the min(k, n) nearest points to (qx, qy).
 *   out_ids [k] int64 device, out_d2 [k] int64 device (may be NULL), n_out HOST = min(k, n).
 * Errors: INVALID_ARG (k < 0, NULL pointers), COORD_RANGE (query or a point out of range),
 * OOM, CUDA.  Synchronises `stream`. */
SPADE_API int spade_knn(const int32_t* xy, int64_t n, int64_t point_id_base, int32_t qx, int32_t qy, int64_t k,
              int64_t* out_ids, int64_t* out_d2, int64_t* n_out, spade_stream_t stream);

/* Probe-path tuning (A/B runs and tests; results never depend on it).  Sets option `name` for
 * this process; returns INVALID_ARG for an unknown name or value.  Initial values come from the
 * environment variable SPADE_<NAME> (upper case), else the default:
 *   "defer"        0 (default) / 1: boundary points always go to the deferral kernel
 *                  (no in-loop warp queues)
 *   "count_global" 0 (default) / 1: COUNT with global counters even when the per-polygon
 *                  shared-memory histogram fits
 *   "global_queue" 0 (default) / 1: in-loop exact tests also for global-counter COUNT
 *   "cache_slots"  4096 (default): max shared-memory count-cache slots of global-counter COUNT
 *                  (power of 2 >= 1024, or 0 = no cache)
 *   "coop"         0 (default, off) / -1 (auto) / 4 / 8 / 16: lanes per deferred point in
 *                  COUNT's cooperative exact-test kernel (measured slower than one point per
 *                  thread on C5 / dj2: fewer points in flight)
 *   "pipe"         -1 (default, auto: > 50% mixed tiles and a per-polygon histogram that would
 *                  fill shared memory) / 0 / 1: COUNT with the cp.async-pipelined probe
 *                  (fine-pixel gathers staged in shared memory, global counters)
 *   "debug_defer"  0 (default) / 1: print deferral statistics to stderr (synchronises)
 *   "defer_xy"     0 (default) / 1: the pipelined probe's deferral entries carry the point
 *                  (re-read from L2 at classification) instead of k_deferred re-reading it
 *                  (measured neutral on C5 / dj2: 11.6 vs 11.6-12.3 ms)
 *   "l2_frac_pct"  100 (default) / 1..100: percent of the fine-canvas lines (by address) gathered
 *                  with L2::evict_last, the rest evict_unchanged (measured: 50/25/12 neutral on
 *                  C5, 1-5% slower on C4 / dj)
 *   "multi_agg"    1 (default) / 0: COUNT counts points on multi-owner pixels (overlapping
 *                  polygons, no edge in the pixel) once per pixel record and spreads the record
 *                  counts over the owner sets afterwards (the paper's partial-aggregate plan,
 *                  P:214), instead of one increment per (point, polygon)
 *   "k_agg"        -1 (default, auto: owner-set entries > 1/2 per record) / 0 / 1: COUNT counts
 *                  boundary points once per pixel record for the record's corner set K (spread
 *                  over K afterwards) plus a +1 / -1 per polygon of odd edge parity, instead of
 *                  merging K per point
 *   "host_chunk"   2^25 (default): points per staging chunk of the host-resident calls
 *                  (256 .. 2^28)
 *   "fine16"       1 (default) / 0: probe canvases that have a 16-bit second level
 *                  (SPADE_CANVAS_NO_FINE16 not set) through it, or through the int32 level
 *   "tma"          0 (default) / 1: COUNT with in-loop exact tests streams the points by TMA bulk
 *                  copies (cp.async.bulk + one mbarrier per warp, 1 KB per warp per batch staged
 *                  in shared memory) instead of 256-bit loads (A/B; measured in profiles/r02)
 *   "smem_pad_kb"  0 (default) .. 64: unused dynamic shared memory added to probe launches (to
 *                  compare variants at an equal shared-memory footprint)
 *   "pipe_notile"  0 (default) / 1: canvases whose coarse tiles are all mixed use the pipelined
 *                  probe without the tile grid, with a full per-polygon histogram in its place
 *                  (measured slower on C5: 13.6 vs 11.2 ms; A/B only)
 *   "hist_copies_max"  16 (default), 32, 8, 4, 2, 1: most copies of the COUNT shared-memory
 *                  histogram (copy = lane mod copies; 32 = one bank per lane, no conflicts)
 *   "idx_queue"    -1 (default) / 0 / 1: COUNT in-loop queues of 4-B point indices instead of 8-B
 *                  points: -1 = for K-aggregated (overlap-heavy) canvases when that keeps the CTA
 *                  at or below the 164 KB shared-memory step (a larger L1 for their record walks:
 *                  ov 29.2 -> 27.1 ms), point queues otherwise (C3 1.69 vs 1.88 ms with index
 *                  queues); 0 = always point queues; 1 = index queues whenever they fit
 *   "stage_events" 0 (default) / 1: record CUDA events between the stages of every COUNT / SELECT /
 *                  PAIRS call on its stream (synchronises once per sub-launch to read them; see
 *                  spade_last_call_stages)
 *   "max_launch_points"  2^31 - 64 (default, the maximum): points per probe sub-launch; a call
 *                  with more points runs several sub-launches (each < 2^31 points: 32-bit point
 *                  offsets and per-record counters; the counters are spread over the owner sets
 *                  after every sub-launch).  Small values (>= 256) exercise the split in tests.
 *   "defer_budget_mb"  4096 (default): device scratch per sub-launch for deferred boundary
 *                  points (16 B per reserved entry; reserved: (2 fb + 4%) of the points, fb = the
 *                  canvas's boundary-pixel fraction).  Calls whose reservation would exceed it
 *                  are cut into more sub-launches, so the peak scratch of spade_join_count /
 *                  spade_select / spade_join_pairs is <= this budget + ~0.2 GB of output
 *                  overflow and compaction tables, whatever n is (64 .. 2^20). */
SPADE_API int spade_set_option(const char* name, int64_t value);

/* Per-stage device time (ms) of this thread's last spade_join_count / spade_select /
 * spade_join_pairs call, recorded when option "stage_events" is 1 (zeros otherwise), summed over
 * its sub-launches: [0] probe kernel (stream, classify, in-loop exact tests, direct sinks),
 * [1] deferred exact tests, [2] output compaction (SELECT / PAIRS), [3] per-record counter
 * expansion (COUNT over overlapping polygons).  Writes min(cap, 4) values; returns 4. */
SPADE_API int spade_last_call_stages(float* ms, int32_t cap);

/* Number of kernels this library has launched in this process (for the bench's gpu_launches). */
SPADE_API int64_t spade_launch_count(void);

SPADE_API const char* spade_status_string(int code);
SPADE_API const char* spade_last_error(void);   /* thread-local detail message of the last failure */

#ifdef __cplusplus
}
#endif
#endif /* SPADE_H */
