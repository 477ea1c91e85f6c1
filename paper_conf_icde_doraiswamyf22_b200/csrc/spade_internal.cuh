// spade_internal.cuh — shared declarations of the CUDA path (canvas layout, exact integer helpers).
// Nothing here is shared with oracle/ (which has its own plain C implementation).
#pragma once

#include <cstdint>
#include <cuda_runtime.h>
#include "../../include/spade.h"

namespace spade {

// ---- canvas encoding ------------------------------------------------------------------------
// Fine canvas pixel (int32), the paper's discrete-canvas pixel (v0, vb) of P:111 reduced to the
// polygon primitive:  v >= 0  -> the single polygon owning the whole (closed) pixel
//                     v == -1 -> no polygon
//                     v <= -2 -> record id  -2 - v  (a boundary pixel, or a multi-owner pixel)
constexpr int32_t kEmpty = -1;
constexpr int32_t kMultiMark = INT32_MIN;     // transient during the fill only
// Coarse (shared-memory) tile entry, uint16: 0 = empty, owner+1 for a uniform tile, and a mixed
// tile is >= mix_min.  Dense layout (mix_min = 0xFFFF): the fine pixel is fine[fy*W + fx].
// Compact layout (mix_min = 0x8000, needs P < 32767 and < 32768 mixed tiles): entry 0x8000|m and
// the tile's pixels are the m-th block of 2^b x 2^b int32 in cfine (only mixed tiles stored).
constexpr uint16_t kTileEmpty = 0, kTileMixed = 0xFFFF, kTileMixedCompact = 0x8000;
// 16-bit copy of a dense fine canvas (P < 65534): code = owner id (< 0xFFFE), kF16Empty, or
// kF16Record (boundary / multi-owner pixel: the record is found through the int32 canvas).
constexpr uint16_t kF16Empty = 0xFFFE, kF16Record = 0xFFFF;

// Boundary-index record as the build derives it (build intermediate; packed into Rec below).
// For a boundary pixel: the distinct polygons whose edges touch the
// closed pixel, rec_polys[poly_begin, +poly_cnt) (ascending), the de-duplicated edges
// [edge_begin, +edge_cnt) in run_seg with run_mask = XOR of (1 << local polygon index) over the
// polygons using that segment (an edge shared by two polygons is stored once; poly_cnt > 64:
// run_mask holds one local index per edge, no merging), and the corrected corner set K (`term`;
// DESIGN.md "Canvas").  For a multi-owner non-boundary pixel: no edges, term = its owner set.
// term >= 0: {term};  term == -1: {};  term <= -2: set m = -2 - term (sets/set_rng).
struct RunRec {
  int64_t edge_begin;
  int32_t edge_cnt;
  int32_t term;
  int32_t poly_begin;
  int32_t poly_cnt;
};
constexpr int kMaskPolys = 64;     // records with more distinct polygons use the slow path

// Packed records: one contiguous blob per record in CanvasDev::blob (16-byte units), located by
// its header's unit offset u, which is what the fine canvas holds for a boundary / multi-owner
// pixel (v = -2 - u).  Layout at u:
//   header (16 B): RecHdr {term, ecnt, pinfo, id}
//   int32 polys[pcnt]                      (padded to 16 B)
//   primitives[ecnt]: short4 (ax,ay,bx,by) relative to the pixel's lower-left corner when every
//                     coordinate fits in int16 (kRecShort), else int4 absolute
//   masks[ecnt]:      uint8 when pcnt <= 8 (kRecByte), else uint64 (toggle mask / local index)
// Multi-owner records (no edges) are a header only, after every boundary record, one unit each.
// `Rec` is the decoded header with `blob` = the data's unit offset (u + 1); the canvas keeps a
// Rec array indexed by record id (= RecHdr::id) for the per-record counter expansion.
struct Rec {
  uint32_t blob;
  int32_t term;
  int32_t ecnt;
  uint32_t pinfo;             // pcnt | kRecShort | kRecByte
};
constexpr uint32_t kRecShort = 1u << 31, kRecByte = 1u << 30, kRecPcnt = (1u << 30) - 1u;

// Canvas kinds: the constraint primitives a canvas is built from (Sec. 4.2).
//   kPolygons: record "edges" are polygon edges (ax, ay, bx, by), exact test = local crossing parity
//   kDisks:    record "edges" are disks (cx, cy, r2 low 32 bits, r2 high 32 bits), exact test =
//              (px-cx)^2 + (py-cy)^2 <= r2 (closed disk, P:127 distance canvases)
constexpr int32_t kPolygons = 0, kDisks = 1;

__host__ __device__ __forceinline__ int64_t disk_r2(int4 e) {
  return (int64_t)((uint64_t)(uint32_t)e.z | ((uint64_t)(uint32_t)e.w << 32));
}

struct CanvasDev {            // passed by value to kernels
  int32_t minx, miny;         // extent origin
  uint32_t extw, exth;        // maxx - minx, maxy - miny (points with larger offsets are outside)
  int32_t s;                  // log2 pixel size
  int32_t W, H;               // fine canvas size (padded to whole tiles: W = Wc << b)
  int32_t b;                  // log2 tile size in fine pixels
  int32_t Wc, Hc;             // coarse grid; the smem array has pitch Wc + 1 and Hc + 1 rows
                              // (last column and row: always-empty sentinel tiles)
  int32_t num_polys;
  int32_t compact;            // 1: compact fine layout (cfine), 0: dense (fine)
  uint32_t mix_min;           // tile entries >= mix_min are mixed
  const int32_t* fine;        // dense W x H canvas (always present)
  const uint16_t* fine16;     // 16-bit copy of it (f16 layout only; see kF16Record)
  int32_t f16;                // 1: the probe's second level is fine16 (dense layout, P < 65534)
  const int32_t* cfine;       // compact mixed-tile blocks (compact layout only)
  const uint16_t* coarse;
  const Rec* recs;            // records: boundary pixels, then multi-owner pixels
  const uint4* blob;          // packed record data (Rec::blob)
  const int32_t* sets;        // concatenated sorted owner sets
  const int2* set_rng;        // (begin, count)
  const uint64_t* kbits;      // per record id: bit k = the record's k-th polygon is in its corner set K (<= 64 polygons)
  int32_t kind;               // kPolygons / kDisks
};

}  // namespace spade

struct spade_canvas {
  spade::CanvasDev d;
  int device = 0;
  bool empty = true;          // no polygon vertices: everything is outside
  int64_t num_runs = 0, num_records = 0, num_run_edges = 0, num_set_entries = 0;
  int64_t num_set_ranges = 0, cfine_elems = 0, coarse_elems = 0;   // array sizes (checksum)
  int64_t multi_unit = 0;     // blob offset of the first multi-owner record header
  float stage_ms[8] = {};     // build stage times (CUDA events on the build stream; spade_canvas_build_times)
  int num_stages = 0;
  double mixed_tile_frac = 0.0;
  // owned device allocations
  int32_t* fine = nullptr;
  uint16_t* fine16 = nullptr;
  int32_t* cfine = nullptr;
  uint16_t* coarse = nullptr;
  spade::Rec* recs = nullptr;
  uint4* blob = nullptr;
  int64_t blob_bytes = 0;
  int32_t* sets = nullptr;
  int2* set_rng = nullptr;
  uint64_t* kbits = nullptr;
  spade::CanvasDev* d_dev = nullptr;   // copy of d in device memory (out-of-line exact test)
};

namespace spade {

// Canvas build stages (timed with CUDA events, NVTX ranges "spade_build:<name>")
constexpr int kBuildStages = 6;
extern const char* const kBuildStageNames[kBuildStages];

// Fine pixel index of pixel (fx, fy) whose coarse tile entry is the mixed value t.
__host__ __device__ __forceinline__ const int32_t* fine_ptr(const CanvasDev& cv, uint32_t t, uint32_t fx, uint32_t fy) {
  if (cv.compact) {
    const uint32_t bm = (1u << cv.b) - 1u;
    return cv.cfine + ((((t & 0x7fffu) << cv.b) | (fy & bm)) << cv.b | (fx & bm));
  }
  return cv.fine + ((size_t)fy * (uint32_t)cv.W + fx);
}

// ---- exact integer helpers (host + device) --------------------------------------------------
__host__ __device__ __forceinline__ int64_t floor_div(int64_t a, int64_t b) {
  int64_t q = a / b, r = a % b;
  return (r != 0 && ((r < 0) != (b < 0))) ? q - 1 : q;
}
__host__ __device__ __forceinline__ int64_t ceil_div(int64_t a, int64_t b) { return -floor_div(-a, b); }

// error plumbing (spade_api.cu)
int set_error(int code, const char* fmt, ...);
int check_cuda(cudaError_t e, const char* what);
void count_launch(int n = 1);
int device_sm_count();
void keep_pool_memory();    // the device's default pool keeps freed memory (probe scratch, build temporaries)

// probe-path options (spade_set_option; include/spade.h)
struct Options {
  int defer, count_global, global_queue, cache_slots, coop, debug_defer, pipe, defer_xy, l2_frac_pct, multi_agg, k_agg;
  int64_t host_chunk;         // points per staging chunk of the host-resident calls
  int64_t max_launch_points;  // points per probe sub-launch (< 2^31; smaller values: tests)
  int64_t defer_budget_mb;    // deferral scratch per sub-launch (16 B per reserved entry)
  int fine16;                 // probe fine16 canvases through their 16-bit level (1) or the int32 one (0)
  int stage_events;           // record per-stage CUDA events in every probe call (spade_last_call_stages)
  int tma;                    // COUNT with in-loop queues: point stream staged by TMA bulk copies (A/B)
  int smem_pad_kb;            // unused dynamic shared memory added to probe launches (equal-footprint A/B)
  int tma_slack_kb;           // "tma": shared memory the TMA variant may use above the 196 KB budget
  int pipe_notile;            // all-mixed canvases: the tile-less pipelined probe with a full histogram
  int hist_copies_max;        // COUNT shared-memory histogram copies, at most (power of 2, <= 32)
  int idx_queue;              // COUNT in-loop queues of point indices: -1 auto, 0 never, 1 always
};
constexpr int kProbeStages = 4;   // probe, deferred exact tests, output compaction, counter expansion
int last_call_stages(float* ms, int cap);

// Makes the canvas's device current for the duration of an entry point (restored after).
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) == cudaSuccess && prev != dev) cudaSetDevice(dev);
    else prev = -1;
  }
  ~DeviceGuard() { if (prev >= 0) cudaSetDevice(prev); }
};
Options& options();

// A forced canvas grid: the polygon x polygon join lays both polygon sets on one pixel grid
// (the extent must contain the set's own; s = log2 pixel, b = log2 tile).
struct GridSpec {
  int32_t minx, miny, maxx, maxy;
  int32_t s, b;
};
int build_canvas_on_grid(const int32_t* ring_xy, const int64_t* ring_off, const int64_t* poly_ring_off, int32_t P,
                         const GridSpec& grid, cudaStream_t st, spade_canvas** out);
// tile exponent the builder picks for a W0 x H0 pixel canvas over P polygons
int tile_log2_for(int64_t W0, int64_t H0, int32_t P);

// probe launchers (probe.cu)
int launch_count(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t* counts, cudaStream_t st);
int launch_select(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t base, int64_t* out,
                  int64_t cap, unsigned long long* d_total, cudaStream_t st);
int launch_pairs(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t base, int64_t* opt,
                 int32_t* opl, int64_t cap, unsigned long long* d_total, cudaStream_t st);

// kNN (knn.cu): squared-distance buckets = concentric circles of the paper's kNN plan
constexpr int kKnnBins = 248;      // == SPADE_KNN_BINS
uint64_t knn_bucket_r2(int b);
int knn_hist(const int32_t* xy, int64_t n, int32_t qx, int32_t qy, int64_t* hist, cudaStream_t st);
int knn_select(const int32_t* xy, int64_t n, int64_t base, int32_t qx, int32_t qy, uint64_t r2, int64_t* out_ids,
               int64_t* out_d2, int64_t cap, unsigned long long* d_total, cudaStream_t st);
int knn_topk(const int64_t* ids, const int64_t* d2, int64_t m, int64_t k, int64_t* out_ids, int64_t* out_d2,
             cudaStream_t st);

}  // namespace spade
