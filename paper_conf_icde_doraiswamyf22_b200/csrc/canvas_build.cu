// canvas_build.cu — spade_build_canvas: exact integer rasterisation of polygons into the discrete
// canvas + boundary index (Sec. 4.2 canvas creation P:113-123, Sec. 4.3 boundary index
// P:140-146, Sec. 5.5 boundary-index creation P:268).  Replaces the paper's OpenGL pipeline
// (triangulation P:117, two-pass triangle/line render P:121, conservative rasterisation P:123)
// with data-parallel kernels:
//   K-B0  edges of all rings (+ polygon id), coordinate range check, extent
//   K-B1  edge -> (row, pixel-range) fragments of every CLOSED pixel an edge touches (exact
//         rationals), and scanline crossing events at every row's bottom line y = Y0_j
//   K-B2  mark boundary pixels; number them; pixel-local edge lists sorted by polygon
//   K-B3  corner owner sets: per (row, polygon) consecutive event pairs bound the pixels whose
//         lower-left corner lies inside (all pixels, boundary or not); overlaps -> owner sets
//   K-B4  per boundary pixel: K = corner set XOR {polygons whose local edges cross the upward
//         ray from the corner an odd number of times}; records; final canvas encoding
//   K-B5  coarse tile summary (uniform owner / empty / mixed) for the shared-memory level
// The exactness argument: for p in boundary pixel (i, j) with lower-left
// corner c = (X, Y0),  inside(p, P) = [P in K] XOR  (sum over P's local edges of
//          cu(X, py) ^ cr(X, py) ^ cr(px, py))
// where cr / cu are the half-open rightward / upward ray tests (perturbation reading of C1).
#include <cub/cub.cuh>
#include <thrust/iterator/transform_iterator.h>
#include <nvtx3/nvToolsExt.h>
#include <vector>
#include <algorithm>
#include "spade_internal.cuh"

namespace spade {

const char* const kBuildStageNames[kBuildStages] = {
    "edges+extent (K-B0)",        "fragments+events (K-B1)",  "boundary pixels+local edges (K-B2)",
    "corner owner sets (K-B3)",   "K sets+records (K-B4/B6)", "coarse tiles+compact+fine16 (K-B5)"};

namespace {

// CUDA events at the stage boundaries of one build (read after the build's final sync) and an
// NVTX range per stage
struct StageTimer {
  cudaEvent_t ev[kBuildStages + 1] = {};
  int n = 0;
  cudaStream_t st;
  explicit StageTimer(cudaStream_t s) : st(s) {}
  void mark() {                                   // end of the previous stage / start of the next
    if (n > kBuildStages) return;
    if (n > 0) nvtxRangePop();
    if (cudaEventCreate(&ev[n]) == cudaSuccess) cudaEventRecord(ev[n], st);
    if (n < kBuildStages) {
      char name[96];
      snprintf(name, sizeof(name), "spade_build:%s", kBuildStageNames[n]);
      nvtxRangePushA(name);
    }
    ++n;
  }
  void read(float* out, int* count) {             // after a sync of st
    *count = 0;
    for (int i = 0; i + 1 < n; ++i) {
      float ms = 0.f;
      if (ev[i] && ev[i + 1] && cudaEventElapsedTime(&ms, ev[i], ev[i + 1]) == cudaSuccess) out[i] = ms;
      *count = i + 1;
    }
  }
  ~StageTimer() {
    if (n > 0 && n <= kBuildStages) nvtxRangePop();
    for (cudaEvent_t e : ev)
      if (e) cudaEventDestroy(e);
  }
};

struct Geo {
  int64_t minx, miny;
  int s;
  int64_t S;
  int W, H;
};

constexpr int kBT = 256;

__host__ __device__ __forceinline__ int64_t imax64(int64_t a, int64_t b) { return a > b ? a : b; }
__host__ __device__ __forceinline__ int64_t imin64(int64_t a, int64_t b) { return a < b ? a : b; }

__device__ __forceinline__ int64_t upper_bound_i64(const int64_t* a, int64_t n, int64_t v) {
  int64_t lo = 0, hi = n;  // first index with a[idx] > v
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (a[mid] <= v) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// K-B0: one edge per vertex (vertex k -> next vertex of its ring), its polygon, range check, extent
__global__ void k_edges(const int2* __restrict__ xy, const int64_t* __restrict__ ring_off, int64_t R,
                        const int64_t* __restrict__ poly_ring_off, int32_t P, int64_t V,
                        int4* __restrict__ seg, int32_t* __restrict__ poly, int* __restrict__ ext,
                        int* __restrict__ bad) {
  using BR = cub::BlockReduce<int, kBT>;
  __shared__ typename BR::TempStorage tmp;
  int mnx = INT_MAX, mny = INT_MAX, mxx = INT_MIN, mxy = INT_MIN, b = 0;
  for (int64_t k = blockIdx.x * (int64_t)kBT + threadIdx.x; k < V; k += (int64_t)gridDim.x * kBT) {
    int64_t r = upper_bound_i64(ring_off, R + 1, k) - 1;
    int32_t p = (int32_t)(upper_bound_i64(poly_ring_off, (int64_t)P + 1, r) - 1);
    int64_t k2 = (k + 1 < ring_off[r + 1]) ? k + 1 : ring_off[r];
    int2 a = xy[k], c = xy[k2];
    seg[k] = make_int4(a.x, a.y, c.x, c.y);
    poly[k] = p;
    const int lim = 1 << 30;
    if (a.x < -lim || a.x >= lim || a.y < -lim || a.y >= lim) b = 1;
    mnx = min(mnx, a.x); mny = min(mny, a.y); mxx = max(mxx, a.x); mxy = max(mxy, a.y);
  }
  int r0 = BR(tmp).Reduce(mnx, cub::Min()); __syncthreads();
  int r1 = BR(tmp).Reduce(mny, cub::Min()); __syncthreads();
  int r2 = BR(tmp).Reduce(mxx, cub::Max()); __syncthreads();
  int r3 = BR(tmp).Reduce(mxy, cub::Max()); __syncthreads();
  int r4 = BR(tmp).Reduce(b, cub::Max());
  if (threadIdx.x == 0) {
    atomicMin(&ext[0], r0); atomicMin(&ext[1], r1); atomicMax(&ext[2], r2); atomicMax(&ext[3], r3);
    if (r4) atomicOr(bad, 1);
  }
}

__device__ __forceinline__ bool degenerate(int4 e) { return e.x == e.z && e.y == e.w; }

// rows j whose CLOSED strip [Y0_j, Y0_j + S] meets the edge's y-range
__device__ __forceinline__ void frag_rows(int4 e, const Geo& g, int64_t& jlo, int64_t& jhi) {
  int64_t ylo = imin64(e.y, e.w), yhi = imax64(e.y, e.w);
  jlo = imax64(ceil_div(ylo - g.miny, g.S) - 1, 0);
  jhi = imin64(floor_div(yhi - g.miny, g.S), g.H - 1);
}

// rows j whose bottom line y = Y0_j is straddled half-open: min(a.y,b.y) <= Y0_j < max(a.y,b.y)
__device__ __forceinline__ void event_rows(int4 e, const Geo& g, int64_t& jlo, int64_t& jhi) {
  int64_t ylo = imin64(e.y, e.w), yhi = imax64(e.y, e.w);
  jlo = imax64(ceil_div(ylo - g.miny, g.S), 0);
  jhi = imin64(ceil_div(yhi - g.miny, g.S) - 1, g.H - 1);
}

// closed pixel columns [ilo, ihi] the edge touches inside the closed strip of row j (exact)
__device__ __forceinline__ void frag_cols(int4 e, const Geo& g, int64_t j, int& ilo, int& ihi) {
  int64_t xl, xr;
  if (e.y == e.w) {
    xl = imin64(e.x, e.z); xr = imax64(e.x, e.z);
  } else {
    int64_t ylo = imin64(e.y, e.w), yhi = imax64(e.y, e.w);
    int64_t Y0 = g.miny + j * g.S;
    int64_t ya = imax64(ylo, Y0), yb = imin64(yhi, Y0 + g.S);
    int64_t dx = (int64_t)e.z - e.x, dy = (int64_t)e.w - e.y;
    bool inc = (dx >= 0) == (dy > 0) || dx == 0;      // x non-decreasing in y along the edge
    int64_t ylx = inc ? ya : yb, yhx = inc ? yb : ya;  // y where x is smallest / largest
    xl = e.x + ceil_div(dx * (ylx - e.y), dy);          // ceil(x(ylx))
    xr = e.x + floor_div(dx * (yhx - e.y), dy);         // floor(x(yhx))
  }
  ilo = (int)imax64(ceil_div(xl - g.minx, g.S) - 1, 0);
  ihi = (int)imin64(floor_div(xr - g.minx, g.S), g.W - 1);
}

__global__ void k_count(const int4* __restrict__ seg, int64_t E, Geo g, int64_t* __restrict__ nfrag,
                        int64_t* __restrict__ nev) {
  for (int64_t k = blockIdx.x * (int64_t)kBT + threadIdx.x; k < E; k += (int64_t)gridDim.x * kBT) {
    int4 e = seg[k];
    int64_t a, b;
    frag_rows(e, g, a, b);
    nfrag[k] = (!degenerate(e) && b >= a) ? b - a + 1 : 0;   // zero-length edges never cross anything
    event_rows(e, g, a, b);
    nev[k] = (e.y != e.w && b >= a) ? b - a + 1 : 0;
  }
}

struct Frag { int32_t j, ilo, ihi, e; };

// Warp-cooperative loops: every lane owns one task (an edge, a fragment, an event pair) of n_i
// items; tasks of at most kLongTask items are run by their own lane, longer ones by the whole
// warp in turn (lanes split the items), so one long edge / fill span does not serialise its warp
// (the fine-resolution canvases of small polygon sets: C1 at 1-unit pixels).
constexpr int64_t kLongTask = 16;
__device__ __forceinline__ int64_t shfl64(int64_t v, int src) {
  return (int64_t)(((uint64_t)(uint32_t)__shfl_sync(0xffffffffu, (int)(v >> 32), src) << 32) |
                   (uint32_t)__shfl_sync(0xffffffffu, (int)(uint32_t)v, src));
}
__device__ __forceinline__ int4 shfl4(int4 v, int src) {
  return make_int4(__shfl_sync(0xffffffffu, v.x, src), __shfl_sync(0xffffffffu, v.y, src),
                   __shfl_sync(0xffffffffu, v.z, src), __shfl_sync(0xffffffffu, v.w, src));
}

// one fragment of edge k at row j (closed pixels [ilo, ihi] it touches)
__device__ __forceinline__ void emit_frag(int4 e, int32_t k, const Geo& g, int64_t j, int64_t o, Frag* frags, int64_t* frag_w) {
  int ilo, ihi;
  frag_cols(e, g, j, ilo, ihi);
  frags[o] = Frag{(int32_t)j, ilo, ihi, k};
  frag_w[o] = ihi >= ilo ? ihi - ilo + 1 : 0;
}
// event key: row | polygon | k,  k = 2c + (x* strictly inside column c ? 1 : 0), c = column of x*,
// so that  x* > X_i  <=>  k > 2i  for every column i.
__device__ __forceinline__ uint64_t event_key(int4 e, uint64_t pk, const Geo& g, int64_t j, int pbits, int kbits) {
  const int64_t dx = (int64_t)e.z - e.x, dy = (int64_t)e.w - e.y;
  const int64_t Y0 = g.miny + j * g.S;
  const int64_t t = dx * (Y0 - e.y);
  const int64_t xf = e.x + floor_div(t, dy);                  // floor of the crossing x*
  const int64_t c = floor_div(xf - g.minx, g.S);              // pixel column holding x*
  const bool exact = (t % dy == 0) && ((xf - g.minx) % g.S == 0);
  const uint64_t kk = 2 * (uint64_t)c + (exact ? 0 : 1);
  return ((uint64_t)j << (pbits + kbits)) | (pk << kbits) | kk;
}

__global__ void k_emit(const int4* __restrict__ seg, const int32_t* __restrict__ poly, int64_t E, Geo g,
                       const int64_t* __restrict__ frag_off, const int64_t* __restrict__ ev_off,
                       Frag* __restrict__ frags, int64_t* __restrict__ frag_w, uint64_t* __restrict__ ev_keys,
                       int pbits, int kbits) {
  const int lane = threadIdx.x & 31;
  for (int64_t kb = blockIdx.x * (int64_t)kBT + (threadIdx.x & ~31); kb < E; kb += (int64_t)gridDim.x * kBT) {
    const int64_t k = kb + lane;
    const bool act = k < E;
    const int4 e = act ? seg[k] : make_int4(0, 0, 0, 0);
    int64_t fa = 0, fb = -1, ea = 0, eb = -1, fo = 0, eo = 0;
    uint64_t pk = 0;
    if (act && !degenerate(e)) { frag_rows(e, g, fa, fb); fo = frag_off[k]; }
    if (act && e.y != e.w) { event_rows(e, g, ea, eb); eo = ev_off[k]; pk = (uint64_t)poly[k]; }
    const int64_t nf = fb >= fa ? fb - fa + 1 : 0, ne = eb >= ea ? eb - ea + 1 : 0;
    if (nf <= kLongTask)
      for (int64_t j = fa; j <= fb; ++j) emit_frag(e, (int32_t)k, g, j, fo + (j - fa), frags, frag_w);
    if (ne <= kLongTask)
      for (int64_t j = ea; j <= eb; ++j) ev_keys[eo + (j - ea)] = event_key(e, pk, g, j, pbits, kbits);
    for (unsigned m = __ballot_sync(0xffffffffu, nf > kLongTask); m; m &= m - 1) {
      const int src = __ffs(m) - 1;
      const int4 es = shfl4(e, src);
      const int64_t a = shfl64(fa, src), b = shfl64(fb, src), o = shfl64(fo, src);
      for (int64_t j = a + lane; j <= b; j += 32) emit_frag(es, (int32_t)(kb + src), g, j, o + (j - a), frags, frag_w);
    }
    for (unsigned m = __ballot_sync(0xffffffffu, ne > kLongTask); m; m &= m - 1) {
      const int src = __ffs(m) - 1;
      const int4 es = shfl4(e, src);
      const int64_t a = shfl64(ea, src), b = shfl64(eb, src), o = shfl64(eo, src);
      const uint64_t pks = (uint64_t)shfl64((int64_t)pk, src);
      for (int64_t j = a + lane; j <= b; j += 32) ev_keys[o + (j - a)] = event_key(es, pks, g, j, pbits, kbits);
    }
  }
}

// ---- distance canvases: disks (cx, cy, r2) -----------------------------------------
// A pixel holds the integer points [X, X+S-1] x [Y0, Y0+S-1].  For the closed disk
// (x-cx)^2 + (y-cy)^2 <= r2 the pixel is INSIDE when all its integer points are in the disk,
// TOUCHED when at least one is, and a boundary pixel when touched but not inside.  Per row both
// sets are column intervals (the disk's slice at height y is [cx - hw(y), cx + hw(y)],
// hw(y) = isqrt(r2 - (y-cy)^2), widest at the y closest to cy and narrowest at the farthest), so a
// disk contributes per row: boundary fragments left and right of the inside interval, and one
// pair of fill events bounding it.  Exact integer arithmetic throughout (r2 < 2^62).

__host__ __device__ __forceinline__ int64_t isqrt64(int64_t v) {   // floor(sqrt(v)), 0 <= v < 2^62
  int64_t r = (int64_t)sqrt((double)v);
  while (r > 0 && r * r > v) --r;
  while ((r + 1) * (r + 1) <= v) ++r;
  return r;
}

// K-D0: disks -> (cx, cy, r2 lo, r2 hi) "edges", range check, extent of their integer points.
// bad: 1 = r2 outside [0, 2^62), 2 = a disk reaches outside [-2^30, 2^30)
__global__ void k_disks(const int2* __restrict__ cxy, const int64_t* __restrict__ r2v, int32_t D,
                        int4* __restrict__ seg, int32_t* __restrict__ poly, int* __restrict__ ext,
                        int* __restrict__ bad) {
  using BR = cub::BlockReduce<int, kBT>;
  __shared__ typename BR::TempStorage tmp;
  int mnx = INT_MAX, mny = INT_MAX, mxx = INT_MIN, mxy = INT_MIN, b = 0;
  for (int64_t k = blockIdx.x * (int64_t)kBT + threadIdx.x; k < D; k += (int64_t)gridDim.x * kBT) {
    const int2 c = cxy[k];
    const int64_t r2 = r2v[k];
    const int64_t lim = 1ll << 30;
    if (r2 < 0 || r2 >= (1ll << 62)) { b = max(b, 1); continue; }
    const int64_t R = isqrt64(r2);
    if (c.x - R < -lim || c.x + R >= lim || c.y - R < -lim || c.y + R >= lim) { b = 2; continue; }
    seg[k] = make_int4(c.x, c.y, (int)(uint32_t)(uint64_t)r2, (int)(uint32_t)((uint64_t)r2 >> 32));
    poly[k] = (int32_t)k;
    mnx = min(mnx, (int)(c.x - R)); mny = min(mny, (int)(c.y - R));
    mxx = max(mxx, (int)(c.x + R)); mxy = max(mxy, (int)(c.y + R));
  }
  int r0 = BR(tmp).Reduce(mnx, cub::Min()); __syncthreads();
  int r1 = BR(tmp).Reduce(mny, cub::Min()); __syncthreads();
  int r2 = BR(tmp).Reduce(mxx, cub::Max()); __syncthreads();
  int r3 = BR(tmp).Reduce(mxy, cub::Max()); __syncthreads();
  int r4 = BR(tmp).Reduce(b, cub::Max());
  if (threadIdx.x == 0) {
    atomicMin(&ext[0], r0); atomicMin(&ext[1], r1); atomicMax(&ext[2], r2); atomicMax(&ext[3], r3);
    if (r4) atomicMax(bad, r4);
  }
}

__device__ __forceinline__ void disk_rows(int4 e, const Geo& g, int64_t R, int64_t& jlo, int64_t& jhi) {
  jlo = imax64(floor_div((int64_t)e.y - R - g.miny, g.S), 0);
  jhi = imin64(floor_div((int64_t)e.y + R - g.miny, g.S), g.H - 1);
}

// row j of disk e: touched columns [t0, t1], inside columns [i0, i1] (empty: i0 > i1)
__device__ __forceinline__ void disk_row(int4 e, const Geo& g, int64_t R, int64_t j, int64_t& t0, int64_t& t1,
                                         int64_t& i0, int64_t& i1) {
  const int64_t cx = e.x, cy = e.y, r2 = disk_r2(e);
  const int64_t Y0 = g.miny + j * g.S, Y1 = Y0 + g.S - 1;
  const int64_t ya = imax64(Y0, cy - R), yb = imin64(Y1, cy + R);
  const int64_t dymin = (ya <= cy && cy <= yb) ? 0 : imin64(ya > cy ? ya - cy : cy - ya, yb > cy ? yb - cy : cy - yb);
  const int64_t hw = isqrt64(r2 - dymin * dymin);
  t0 = imax64(floor_div(cx - hw - g.minx, g.S), 0);
  t1 = imin64(floor_div(cx + hw - g.minx, g.S), g.W - 1);
  const int64_t dymax = imax64(Y0 > cy ? Y0 - cy : cy - Y0, Y1 > cy ? Y1 - cy : cy - Y1);
  i0 = 1; i1 = 0;
  if (dymax <= R) {
    const int64_t hm = isqrt64(r2 - dymax * dymax);
    i0 = imax64(ceil_div(cx - hm - g.minx, g.S), t0);
    i1 = imin64(floor_div(cx + hm - g.minx - g.S + 1, g.S), t1);
  }
}

// two fragments and two fill events per (disk, row)
__global__ void k_dcount(const int4* __restrict__ seg, int64_t E, Geo g, int64_t* __restrict__ nfrag,
                         int64_t* __restrict__ nev) {
  for (int64_t k = blockIdx.x * (int64_t)kBT + threadIdx.x; k < E; k += (int64_t)gridDim.x * kBT) {
    const int4 e = seg[k];
    int64_t a, b;
    disk_rows(e, g, isqrt64(disk_r2(e)), a, b);
    nfrag[k] = b >= a ? 2 * (b - a + 1) : 0;
    nev[k] = nfrag[k];
  }
}

__global__ void k_demit(const int4* __restrict__ seg, int64_t E, Geo g, const int64_t* __restrict__ frag_off,
                        const int64_t* __restrict__ ev_off, Frag* __restrict__ frags, int64_t* __restrict__ frag_w,
                        uint64_t* __restrict__ ev_keys, int pbits, int kbits) {
  for (int64_t k = blockIdx.x * (int64_t)kBT + threadIdx.x; k < E; k += (int64_t)gridDim.x * kBT) {
    const int4 e = seg[k];
    const int64_t R = isqrt64(disk_r2(e));
    int64_t a, b;
    disk_rows(e, g, R, a, b);
    int64_t o = frag_off[k], q = ev_off[k];
    for (int64_t j = a; j <= b; ++j, o += 2, q += 2) {
      int64_t t0, t1, i0, i1;
      disk_row(e, g, R, j, t0, t1, i0, i1);
      int64_t l0 = t0, l1 = t1, r0 = 0, r1 = -1, k0 = 0, k1 = 0;   // boundary [l0,l1] u [r0,r1]
      if (i0 <= i1) { l1 = i0 - 1; r0 = i1 + 1; r1 = t1; k0 = 2 * i0; k1 = 2 * (i1 + 1); }
      frags[o] = Frag{(int32_t)j, (int32_t)l0, (int32_t)l1, (int32_t)k};
      frag_w[o] = l1 >= l0 ? l1 - l0 + 1 : 0;
      frags[o + 1] = Frag{(int32_t)j, (int32_t)r0, (int32_t)r1, (int32_t)k};
      frag_w[o + 1] = r1 >= r0 ? r1 - r0 + 1 : 0;
      const uint64_t hk = ((uint64_t)j << (pbits + kbits)) | ((uint64_t)k << kbits);
      ev_keys[q] = hk | (uint64_t)k0;                   // empty interior: [0, 0) fills nothing
      ev_keys[q + 1] = hk | (uint64_t)k1;
    }
  }
}

__global__ void k_mark(const Frag* __restrict__ frags, int64_t F, int W, int32_t* __restrict__ bflag) {
  const int lane = threadIdx.x & 31;
  for (int64_t tb = blockIdx.x * (int64_t)kBT + (threadIdx.x & ~31); tb < F; tb += (int64_t)gridDim.x * kBT) {
    const int64_t t = tb + lane;
    const Frag f = t < F ? frags[t] : Frag{0, 1, 0, 0};
    const int n = f.ihi - f.ilo + 1;
    int32_t* row = bflag + (int64_t)f.j * W;
    if (n <= kLongTask)
      for (int i = f.ilo; i <= f.ihi; ++i) row[i] = 1;
    for (unsigned m = __ballot_sync(0xffffffffu, n > kLongTask); m; m &= m - 1) {
      const int src = __ffs(m) - 1;
      const int j = __shfl_sync(0xffffffffu, f.j, src), lo = __shfl_sync(0xffffffffu, f.ilo, src),
                hi = __shfl_sync(0xffffffffu, f.ihi, src);
      for (int i = lo + lane; i <= hi; i += 32) bflag[(int64_t)j * W + i] = 1;
    }
  }
}

// bscan = inclusive scan of boundary flags: boundary pixel p has id bscan[p] - 1
__global__ void k_bids(const int32_t* __restrict__ bflag, const int32_t* __restrict__ bscan, int64_t WH,
                       int64_t* __restrict__ pix_of) {
  for (int64_t p = blockIdx.x * (int64_t)kBT + threadIdx.x; p < WH; p += (int64_t)gridDim.x * kBT)
    if (bflag[p]) pix_of[bscan[p] - 1] = p;
}

// one (boundary pixel, edge) entry per pixel of every fragment
__device__ __forceinline__ void local_entry(const int32_t* __restrict__ bscan, int64_t p, int64_t o, uint32_t pk, int32_t e,
                                            uint64_t* __restrict__ keys, int32_t* __restrict__ vals, int32_t* __restrict__ cnt) {
  const int32_t bid = bscan[p] - 1;
  keys[o] = ((uint64_t)(uint32_t)bid << 32) | pk;
  vals[o] = e;
  atomicAdd(&cnt[bid], 1);
}
__global__ void k_local(const Frag* __restrict__ frags, int64_t F, int W, const int64_t* __restrict__ lw_off,
                        const int32_t* __restrict__ poly, const int32_t* __restrict__ bscan,
                        uint64_t* __restrict__ keys, int32_t* __restrict__ vals, int32_t* __restrict__ cnt) {
  const int lane = threadIdx.x & 31;
  for (int64_t tb = blockIdx.x * (int64_t)kBT + (threadIdx.x & ~31); tb < F; tb += (int64_t)gridDim.x * kBT) {
    const int64_t t = tb + lane;
    const bool act = t < F;
    const Frag f = act ? frags[t] : Frag{0, 1, 0, 0};
    const int64_t o = act ? lw_off[t] : 0;
    const uint32_t pk = act ? (uint32_t)poly[f.e] : 0u;
    const int n = f.ihi - f.ilo + 1;
    if (n <= kLongTask)
      for (int i = f.ilo; i <= f.ihi; ++i) local_entry(bscan, (int64_t)f.j * W + i, o + (i - f.ilo), pk, f.e, keys, vals, cnt);
    for (unsigned m = __ballot_sync(0xffffffffu, n > kLongTask); m; m &= m - 1) {
      const int src = __ffs(m) - 1;
      const int j = __shfl_sync(0xffffffffu, f.j, src), lo = __shfl_sync(0xffffffffu, f.ilo, src),
                hi = __shfl_sync(0xffffffffu, f.ihi, src), es = __shfl_sync(0xffffffffu, f.e, src);
      const int64_t os = shfl64(o, src);
      const uint32_t pks = (uint32_t)__shfl_sync(0xffffffffu, (int)pk, src);
      for (int i = lo + lane; i <= hi; i += 32) local_entry(bscan, (int64_t)j * W + i, os + (i - lo), pks, es, keys, vals, cnt);
    }
  }
}

// --- pixel-local edge de-duplication (an edge shared by two polygons, or used twice, is stored
// once with a polygon toggle mask) ---------------------------------------------------------------
// entries sorted by (bid, poly): head of each distinct (bid, poly)
__global__ void k_iota(int32_t* __restrict__ a, int64_t n) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < n; t += (int64_t)gridDim.x * kBT) a[t] = (int32_t)t;
}

__global__ void k_polyhead(const uint64_t* __restrict__ key, int64_t L, int32_t* __restrict__ head) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < L; t += (int64_t)gridDim.x * kBT)
    head[t] = (t == 0 || key[t] != key[t - 1]) ? 1 : 0;
}

// pg = inclusive scan of head: distinct (bid, poly) index pg - 1; per-record polygon range
__global__ void k_recpolys(const uint64_t* __restrict__ key, int64_t L, const int32_t* __restrict__ head,
                           const int32_t* __restrict__ pg, int32_t* __restrict__ rec_polys) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < L; t += (int64_t)gridDim.x * kBT)
    if (head[t]) rec_polys[pg[t] - 1] = (int32_t)(key[t] & 0xffffffffu);
}

__global__ void k_polyrange(int64_t NB, const int64_t* __restrict__ le_beg, const int32_t* __restrict__ le_cnt,
                            const int32_t* __restrict__ pg, int32_t* __restrict__ pbeg, int32_t* __restrict__ pcnt) {
  for (int64_t b = blockIdx.x * (int64_t)kBT + threadIdx.x; b < NB; b += (int64_t)gridDim.x * kBT) {
    const int32_t n = le_cnt[b];
    if (n == 0) { pbeg[b] = 0; pcnt[b] = 0; continue; }
    const int64_t e0 = le_beg[b];
    pbeg[b] = pg[e0] - 1;
    pcnt[b] = pg[e0 + n - 1] - pg[e0] + 1;
  }
}

__device__ __forceinline__ uint32_t seg_hash(int4 e) {
  // canonical orientation, then a 64-bit mix folded to 32 bits
  int ax = e.x, ay = e.y, bx = e.z, by = e.w;
  if (bx < ax || (bx == ax && by < ay)) { int t = ax; ax = bx; bx = t; t = ay; ay = by; by = t; }
  uint64_t h = ((uint64_t)(uint32_t)ax << 32 | (uint32_t)ay) * 0x9E3779B97F4A7C15ull;
  h ^= ((uint64_t)(uint32_t)bx << 32 | (uint32_t)by) + 0x632BE59BD9B4E019ull + (h << 6) + (h >> 2);
  h ^= h >> 29; h *= 0xBF58476D1CE4E5B9ull; h ^= h >> 32;
  return (uint32_t)h;
}
// equal primitives: a polygon edge in either orientation; a disk exactly
__device__ __forceinline__ bool same_seg(int4 a, int4 b, int kind) {
  return (a.x == b.x && a.y == b.y && a.z == b.z && a.w == b.w) ||
         (kind == kPolygons && a.x == b.z && a.y == b.w && a.z == b.x && a.w == b.y);
}

// per entry (sorted by (bid, poly)): local polygon index and the (bid, segment hash) key
__global__ void k_segkey(const uint64_t* __restrict__ key, const int32_t* __restrict__ ev, int64_t L,
                         const int4* __restrict__ seg, const int32_t* __restrict__ pg, const int32_t* __restrict__ pbeg,
                         uint64_t* __restrict__ key2, int32_t* __restrict__ li) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < L; t += (int64_t)gridDim.x * kBT) {
    const uint32_t bid = (uint32_t)(key[t] >> 32);
    li[t] = pg[t] - 1 - pbeg[bid];
    key2[t] = ((uint64_t)bid << 32) | seg_hash(seg[ev[t]]);
  }
}

// entries sorted by (bid, hash): the first occurrence of each exact segment within its equal-key
// run carries the XOR of the polygon bits of all its occurrences; zero masks (a segment used
// an even number of times by the same polygons) contribute nothing and are dropped.  Records with
// more than kMaskPolys polygons keep every entry with its local index.  PASS 0 flags the kept
// entries (keep[u]) and counts them per record; PASS 1 writes entry u at its rank among the kept
// entries (kpos = exclusive scan of keep: the entries are sorted by record, so a record's kept
// entries start at mbeg[bid]) -- positions independent of thread timing, so the canvas bytes are
// deterministic (spade_canvas_checksum).
template <int PASS>
__global__ void k_merge(const uint64_t* __restrict__ key2, const int32_t* __restrict__ tix, int64_t L,
                        const int32_t* __restrict__ ev, const int32_t* __restrict__ li, const int4* __restrict__ seg,
                        const int32_t* __restrict__ pcnt, const int64_t* __restrict__ le_beg, int32_t* __restrict__ mcnt,
                        const int64_t* __restrict__ mbeg, int32_t* __restrict__ keep, const int64_t* __restrict__ kpos,
                        int4* __restrict__ oseg, uint64_t* __restrict__ omask, int kind) {
  for (int64_t u = blockIdx.x * (int64_t)kBT + threadIdx.x; u < L; u += (int64_t)gridDim.x * kBT) {
    if (PASS == 1 && !keep[u]) continue;
    const uint64_t k = key2[u];
    const uint32_t bid = (uint32_t)(k >> 32);
    const int4 e = seg[ev[tix[u]]];
    uint64_t m;
    const bool slow = pcnt[bid] > kMaskPolys;
    if (slow) {
      m = (uint64_t)li[tix[u]];
    } else {
      bool first = true;
      if (PASS == 0)
        for (int64_t w = u - 1; w >= 0 && key2[w] == k; --w)
          if (same_seg(seg[ev[tix[w]]], e, kind)) { first = false; break; }
      if (!first) { keep[u] = 0; continue; }
      m = 1ull << li[tix[u]];
      for (int64_t w = u + 1; w < L && key2[w] == k; ++w)
        if (same_seg(seg[ev[tix[w]]], e, kind)) m ^= 1ull << li[tix[w]];
      if (m == 0) { if (PASS == 0) keep[u] = 0; continue; }
    }
    if (PASS == 0) {
      keep[u] = 1;
      atomicAdd(&mcnt[bid], 1);
    } else {
      // slow records keep the (bid, poly) order of the entries: grouped by local index
      const int64_t pos = slow ? mbeg[bid] + ((int64_t)tix[u] - le_beg[bid]) : kpos[u];
      oseg[pos] = e;
      omask[pos] = m;
    }
  }
}

// K-B3: sorted events of one (row, polygon) come in consecutive pairs (a closed ring crosses a
// horizontal line an even number of times).  Polygon P contains the lower-left corner of pixel
// i iff 2i lies in [k_a, k_b) for a pair, i.e. i in [ceil(k_a/2), ceil(k_b/2) - 1].
__device__ __forceinline__ void fill_pixel(int32_t* __restrict__ corner, int64_t j, int W, int i, int32_t p,
                                           unsigned long long* __restrict__ multi, unsigned long long* __restrict__ nmulti,
                                           int64_t multi_cap) {
  int32_t* row = corner + j * W;
  const int old = atomicCAS(&row[i], kEmpty, p);
  if (old == kEmpty) return;
  const int prev = atomicExch(&row[i], kMultiMark);
  const unsigned long long q = atomicAdd(nmulti, prev >= 0 ? 2ull : 1ull);
  const uint64_t px = (uint64_t)(j * W + i);
  if ((int64_t)q < multi_cap) multi[q] = (px << 32) | (uint32_t)p;
  if (prev >= 0 && (int64_t)q + 1 < multi_cap) multi[q + 1] = (px << 32) | (uint32_t)prev;
}
__global__ void k_fill(const uint64_t* __restrict__ ev, int64_t NE, int W, int pbits, int kbits,
                       int32_t* __restrict__ corner, unsigned long long* __restrict__ multi,
                       unsigned long long* __restrict__ nmulti, int64_t multi_cap, int* __restrict__ bad) {
  const uint64_t kmask = (1ull << kbits) - 1, pmask = (1ull << pbits) - 1;
  const int64_t NP = NE / 2;
  const int lane = threadIdx.x & 31;
  if (blockIdx.x == 0 && threadIdx.x == 0 && (NE & 1)) atomicOr(bad, 2);
  for (int64_t tb = blockIdx.x * (int64_t)kBT + (threadIdx.x & ~31); tb < NP; tb += (int64_t)gridDim.x * kBT) {
    const int64_t t = tb + lane;
    int64_t j = 0;
    int32_t p = 0;
    int i0 = 0, i1 = 0;
    if (t < NP) {
      const uint64_t k0 = ev[2 * t], k1 = ev[2 * t + 1];
      if ((k0 >> kbits) != (k1 >> kbits)) {
        atomicOr(bad, 2);
      } else {
        j = (int64_t)(k0 >> (kbits + pbits));
        p = (int32_t)((k0 >> kbits) & pmask);
        const int64_t ka = (int64_t)(k0 & kmask), kb = (int64_t)(k1 & kmask);
        i0 = (int)((ka + 1) >> 1); i1 = (int)((kb + 1) >> 1);    // [ceil(ka/2), ceil(kb/2))
      }
    }
    if (i1 - i0 <= kLongTask)
      for (int i = i0; i < i1; ++i) fill_pixel(corner, j, W, i, p, multi, nmulti, multi_cap);
    for (unsigned m = __ballot_sync(0xffffffffu, i1 - i0 > kLongTask); m; m &= m - 1) {
      const int src = __ffs(m) - 1;
      const int64_t js = shfl64(j, src);
      const int32_t ps = __shfl_sync(0xffffffffu, p, src);
      const int a = __shfl_sync(0xffffffffu, i0, src), b = __shfl_sync(0xffffffffu, i1, src);
      for (int i = a + lane; i < b; i += 32) fill_pixel(corner, js, W, i, ps, multi, nmulti, multi_cap);
    }
  }
}

// sorted (pixel << 32 | poly) -> head flags of pixel groups
__global__ void k_multi_heads(const unsigned long long* __restrict__ m, int64_t M, int32_t* __restrict__ head) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < M; t += (int64_t)gridDim.x * kBT)
    head[t] = (t == 0 || (m[t] >> 32) != (m[t - 1] >> 32)) ? 1 : 0;
}

// head_scan = inclusive scan of heads: owner-set index g = head_scan[t] - 1; corner[p] = -2 - g
__global__ void k_multi_sets(const unsigned long long* __restrict__ m, int64_t M, const int32_t* __restrict__ hs,
                             int32_t* __restrict__ sets, int2* __restrict__ set_rng, int32_t* __restrict__ corner) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < M; t += (int64_t)gridDim.x * kBT) {
    int32_t g = hs[t] - 1;
    sets[t] = (int32_t)(m[t] & 0xffffffffu);
    bool head = (t == 0 || (m[t] >> 32) != (m[t - 1] >> 32));
    if (!head) continue;
    int64_t e = t + 1;
    while (e < M && (m[e] >> 32) == (m[t] >> 32)) ++e;
    set_rng[g] = make_int2((int)t, (int)(e - t));
    corner[(int64_t)(m[t] >> 32)] = -2 - g;
  }
}

// half-open upward-ray test at q = (qx, qy) (perturbation reading: ray from (qx+e', qy+e)).
__device__ __forceinline__ int cu_test(int4 e, int64_t qx, int64_t qy) {
  if ((e.x > qx) == (e.z > qx)) return 0;
  int64_t dx = (int64_t)e.z - e.x, dy = (int64_t)e.w - e.y;
  int64_t w = dy * (qx - e.x) - dx * (qy - e.y);
  return dx > 0 ? (w > 0 || (w == 0 && dy > 0)) : (w < 0 || (w == 0 && dy < 0));
}

// K-B4: K = corner set XOR {P : odd number of P's local edges cross the upward ray from the
// corner}.  PASS 0 counts |K| into ksize; PASS 1 writes records and the members of sets with
// |K| >= 2 at kout[koff[b] ...] (ascending polygon order).
template <int PASS>
__global__ void k_kset(int64_t NB, const int64_t* __restrict__ pix_of, Geo g, const int32_t* __restrict__ corner,
                       const int32_t* __restrict__ csets, const int2* __restrict__ crng,
                       const int64_t* __restrict__ mbeg, const int32_t* __restrict__ mcnt,
                       const int4* __restrict__ rseg, const uint64_t* __restrict__ rmask,
                       const int32_t* __restrict__ pbeg, const int32_t* __restrict__ pcnt,
                       const int32_t* __restrict__ rec_polys,
                       int32_t* __restrict__ ksize, const int64_t* __restrict__ koff, int32_t* __restrict__ kout,
                       RunRec* __restrict__ recs, int kind) {
  for (int64_t b = blockIdx.x * (int64_t)kBT + threadIdx.x; b < NB; b += (int64_t)gridDim.x * kBT) {
    const int64_t p = pix_of[b];
    const int64_t i = p % g.W, j = p / g.W;
    const int64_t X = g.minx + i * g.S, Y0 = g.miny + j * g.S;
    const int32_t cv = corner[p];
    int cn, cb = 0;
    if (cv >= 0) cn = 1; else if (cv == kEmpty) cn = 0; else { int2 r = crng[-2 - cv]; cb = r.x; cn = r.y; }
    const bool big = PASS == 1 && ksize[b] >= 2;
    int64_t out = big ? koff[b] : 0;
    int n = 0;
    int32_t first = kEmpty;
    const int64_t e0 = mbeg[b], e1 = e0 + mcnt[b];
    const int32_t pb = pbeg[b], pc = pcnt[b];
    auto put = [&](int32_t Q) {
      if (big) kout[out++] = Q;
      if (n == 0) first = Q;
      ++n;
    };
    int ci = 0;
    auto cel = [&](int k) { return cv >= 0 ? cv : csets[cb + k]; };
    auto merge_upto = [&](int32_t P, int par) {      // corner-set members < P pass through
      while (ci < cn && cel(ci) < P) { put(cel(ci)); ++ci; }
      if (ci < cn && cel(ci) == P) { par ^= 1; ++ci; }
      if (par) put(P);
    };
    if (pc <= kMaskPolys) {
      uint64_t m = 0;
      if (kind == kPolygons)
        for (int64_t e = e0; e < e1; ++e) if (cu_test(rseg[e], X, Y0)) m ^= rmask[e];
      for (int k = 0; k < pc; ++k) {
        const int par = (int)((m >> k) & 1u);
        const int32_t P = rec_polys[pb + k];
        merge_upto(P, par);
      }
    } else {
      for (int k = 0; k < pc; ++k) {
        int par = 0;
        if (kind == kPolygons)
          for (int64_t e = e0; e < e1; ++e) if ((int)rmask[e] == k) par ^= cu_test(rseg[e], X, Y0);
        merge_upto(rec_polys[pb + k], par);
      }
    }
    merge_upto(INT32_MAX, 0);
    if (PASS == 0) ksize[b] = n;
    else recs[b] = RunRec{e0, (int32_t)(e1 - e0), first, pb, pc};   // |K| >= 2 fixed up by k_kset_rng
  }
}

__global__ void k_kset_rng(int64_t NB, const int32_t* __restrict__ ksize, const int64_t* __restrict__ koff,
                           const int32_t* __restrict__ kidx, int64_t base_idx, int64_t base_pos,
                           int2* __restrict__ set_rng, RunRec* __restrict__ recs) {
  for (int64_t b = blockIdx.x * (int64_t)kBT + threadIdx.x; b < NB; b += (int64_t)gridDim.x * kBT) {
    if (ksize[b] < 2) continue;
    int64_t g = base_idx + kidx[b];
    set_rng[g] = make_int2((int)(base_pos + koff[b]), ksize[b]);
    recs[b].term = -2 - (int32_t)g;
  }
}

// final encoding: boundary pixel -> -2 - (its record's header offset in the blob); multi-owner
// corner (owner set g) -> -2 - (record NB + g's header offset)
// per boundary record: which of its local polygons belong to its corner set K (the K-aggregated
// COUNT's sign of a polygon of odd edge parity, without searching K per point)
__global__ void k_kbits(int64_t NR, int64_t NB, const RunRec* __restrict__ runs, const int32_t* __restrict__ rec_polys,
                        const int32_t* __restrict__ sets, const int2* __restrict__ set_rng, uint64_t* __restrict__ kbits) {
  for (int64_t r = blockIdx.x * (int64_t)kBT + threadIdx.x; r < NR; r += (int64_t)gridDim.x * kBT) {
    uint64_t m = 0;
    if (r < NB) {
      const RunRec x = runs[r];
      if (x.poly_cnt <= kMaskPolys && x.term != kEmpty) {
        int tb = 0, tn = 1;
        if (x.term < -1) { const int2 g = set_rng[-2 - x.term]; tb = g.x; tn = g.y; }
        for (int k = 0; k < x.poly_cnt; ++k) {
          const int32_t P = rec_polys[x.poly_begin + k];
          bool in = false;
          if (x.term >= 0) in = P == x.term;
          else { int lo = 0, hi = tn; while (lo < hi) { const int mid = (lo + hi) >> 1; if (sets[tb + mid] < P) lo = mid + 1; else hi = mid; }
                 in = lo < tn && sets[tb + lo] == P; }
          if (in) m |= 1ull << k;
        }
      }
    }
    kbits[r] = m;
  }
}

__global__ void k_finalize(int64_t WH, const int32_t* __restrict__ bflag, const int32_t* __restrict__ bscan,
                           const int32_t* __restrict__ corner, int64_t NB, const int64_t* __restrict__ boff,
                           int32_t* __restrict__ fine) {
  for (int64_t p = blockIdx.x * (int64_t)kBT + threadIdx.x; p < WH; p += (int64_t)gridDim.x * kBT) {
    if (bflag[p]) { fine[p] = (int32_t)(-2 - boff[bscan[p] - 1]); continue; }
    int32_t v = corner[p];
    fine[p] = v >= kEmpty ? v : (int32_t)(-2 - boff[NB + (-2 - (int64_t)v)]);   // owner set g -> record NB + g
  }
}

__global__ void k_multi_recs(int64_t NG, int64_t NB, RunRec* __restrict__ recs) {
  for (int64_t g = blockIdx.x * (int64_t)kBT + threadIdx.x; g < NG; g += (int64_t)gridDim.x * kBT)
    recs[NB + g] = RunRec{0, 0, (int32_t)(-2 - g), 0, 0};
}

// K-B5: tile summary.  tval = owner + 1 / 0 for uniform tiles; mixed tiles flagged in tmix.
__global__ void k_coarse(const int32_t* __restrict__ fine, int W, int H, int b, int Wc, int Hc,
                         int32_t* __restrict__ tval, int32_t* __restrict__ tmix) {
  int64_t NT = (int64_t)Wc * Hc;
  const int B = 1 << b;
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < NT; t += (int64_t)gridDim.x * kBT) {
    int tx = (int)(t % Wc), ty = (int)(t / Wc);
    int i0 = tx * B, j0 = ty * B;
    int i1 = min(i0 + B, W), j1 = min(j0 + B, H);
    int32_t v0 = fine[(int64_t)j0 * W + i0];
    bool uni = v0 >= kEmpty;
    for (int j = j0; j < j1 && uni; ++j)
      for (int i = i0; i < i1; ++i)
        if (fine[(int64_t)j * W + i] != v0) { uni = false; break; }
    tval[t] = uni ? v0 + 1 : -1;
    tmix[t] = uni ? 0 : 1;
  }
}

// coarse entries; compact layout copies each mixed tile's pixels into block m = mscan[t]
__global__ void k_coarse_final(const int32_t* __restrict__ tval, const int32_t* __restrict__ mscan, int Wc, int Hc,
                               int compact, uint32_t owner_lim, uint16_t* __restrict__ coarse) {
  const int64_t NT1 = (int64_t)(Wc + 1) * (Hc + 1);          // with the sentinel column and row
  for (int64_t u = blockIdx.x * (int64_t)kBT + threadIdx.x; u < NT1; u += (int64_t)gridDim.x * kBT) {
    const int tx = (int)(u % (Wc + 1)), ty = (int)(u / (Wc + 1));
    uint16_t e = kTileEmpty;
    if (tx < Wc && ty < Hc) {
      const int64_t t = (int64_t)ty * Wc + tx;
      const int32_t v = tval[t];
      if (v >= 0 && (uint32_t)v < owner_lim) e = (uint16_t)v;
      else e = compact ? (uint16_t)(kTileMixedCompact | (uint32_t)mscan[t]) : kTileMixed;
    }
    coarse[u] = e;
  }
}

__global__ void k_compact(const int32_t* __restrict__ fine, int W, int H, int b, int Wc, const int32_t* __restrict__ tval,
                          const int32_t* __restrict__ mscan, int64_t NT, uint32_t owner_lim, int32_t* __restrict__ cfine) {
  const int B = 1 << b;
  const int64_t NP = NT << (2 * b);
  for (int64_t q = blockIdx.x * (int64_t)kBT + threadIdx.x; q < NP; q += (int64_t)gridDim.x * kBT) {
    const int64_t t = q >> (2 * b);
    const int32_t v = tval[t];
    if (v >= 0 && (uint32_t)v < owner_lim) continue;       // uniform tile: not stored
    const int within = (int)(q & ((1 << (2 * b)) - 1));
    const int i = (int)(t % Wc) * B + (within & (B - 1)), j = (int)(t / Wc) * B + (within >> b);
    cfine[((int64_t)mscan[t] << (2 * b)) + within] = (i < W && j < H) ? fine[(int64_t)j * W + i] : kEmpty;
  }
}

// 16-bit copy of the dense canvas (spade_internal.cuh kF16*)
__global__ void k_fine16(const int32_t* __restrict__ fine, int64_t WH, uint16_t* __restrict__ f16) {
  for (int64_t p = blockIdx.x * (int64_t)kBT + threadIdx.x; p < WH; p += (int64_t)gridDim.x * kBT) {
    const int32_t v = fine[p];
    f16[p] = v >= 0 ? (uint16_t)v : v == kEmpty ? kF16Empty : kF16Record;
  }
}

struct BigSize { __host__ __device__ int64_t operator()(int32_t v) const { return v >= 2 ? v : 0; } };
struct BigFlag { __host__ __device__ int32_t operator()(int32_t v) const { return v >= 2 ? 1 : 0; } };

// K-B6: packed records (spade_internal.cuh "Rec").  Every record is one contiguous blob: a 16-B
// header (RecHdr) followed by its data; the fine canvas holds the header's blob offset, so the
// probe reaches a record's data with no separate record fetch.  Blob size in 16-byte units and
// layout flags: polygon primitives are stored relative to the pixel's lower-left corner as int16
// when all four coordinates fit, masks as bytes when the pixel has <= 8 polygons.  Multi-owner
// records (r >= NB) are a header only: they come last, one unit each (the probe's per-record
// counters are indexed by their unit offset minus the first one's).
__device__ __forceinline__ bool fits16(int64_t v) { return v >= -32768 && v <= 32767; }
__global__ void k_blob_size(int64_t NR, int64_t NB, const RunRec* __restrict__ runs, const int64_t* __restrict__ pix_of,
                            Geo g, const int4* __restrict__ rseg, int kind, int64_t* __restrict__ bsz,
                            uint32_t* __restrict__ bflags) {
  for (int64_t r = blockIdx.x * (int64_t)kBT + threadIdx.x; r < NR; r += (int64_t)gridDim.x * kBT) {
    if (r >= NB) { bsz[r] = 1; bflags[r] = 0; continue; }          // multi-owner record: header only
    const RunRec x = runs[r];
    const int64_t p = pix_of[r];
    const int64_t X = g.minx + (p % g.W) * g.S, Y = g.miny + (p / g.W) * g.S;
    bool sh = kind == kPolygons;
    for (int64_t e = x.edge_begin; e < x.edge_begin + x.edge_cnt && sh; ++e) {
      const int4 q = rseg[e];
      sh = fits16(q.x - X) && fits16(q.y - Y) && fits16(q.z - X) && fits16(q.w - Y);
    }
    const bool by = x.poly_cnt <= 8;
    const int64_t bytes = (((int64_t)x.poly_cnt * 4 + 15) & ~15ll) + (int64_t)x.edge_cnt * ((sh ? 8 : 16) + (by ? 1 : 8));
    bsz[r] = 1 + ((bytes + 15) >> 4);
    bflags[r] = (sh ? kRecShort : 0u) | (by ? kRecByte : 0u);
  }
}

__global__ void k_blob_pack(int64_t NR, int64_t NB, const RunRec* __restrict__ runs, const int64_t* __restrict__ pix_of,
                            Geo g, const int4* __restrict__ rseg, const uint64_t* __restrict__ rmask,
                            const int32_t* __restrict__ rec_polys, const int64_t* __restrict__ boff,
                            const uint32_t* __restrict__ bflags, Rec* __restrict__ recs, uint4* __restrict__ blob) {
  for (int64_t r = blockIdx.x * (int64_t)kBT + threadIdx.x; r < NR; r += (int64_t)gridDim.x * kBT) {
    const RunRec x = runs[r];
    const uint32_t data = (uint32_t)boff[r] + 1u;
    if (r >= NB) {
      recs[r] = Rec{data, x.term, 0, 0u};
      blob[boff[r]] = make_uint4((uint32_t)x.term, 0u, 0u, (uint32_t)r);
      continue;
    }
    const uint32_t fl = bflags[r];
    recs[r] = Rec{data, x.term, x.edge_cnt, (uint32_t)x.poly_cnt | fl};
    blob[boff[r]] = make_uint4((uint32_t)x.term, (uint32_t)x.edge_cnt, (uint32_t)x.poly_cnt | fl, (uint32_t)r);
    unsigned char* b = (unsigned char*)(blob + data);
    int32_t* pp = (int32_t*)b;
    for (int k = 0; k < x.poly_cnt; ++k) pp[k] = rec_polys[x.poly_begin + k];
    unsigned char* eb = b + (((int64_t)x.poly_cnt * 4 + 15) & ~15ll);
    const bool sh = fl & kRecShort, by = fl & kRecByte;
    unsigned char* mb = eb + (int64_t)x.edge_cnt * (sh ? 8 : 16);
    const int64_t p = pix_of[r];
    const int X = (int)(g.minx + (p % g.W) * g.S), Y = (int)(g.miny + (p / g.W) * g.S);
    for (int k = 0; k < x.edge_cnt; ++k) {
      const int4 q = rseg[x.edge_begin + k];
      if (sh) ((short4*)eb)[k] = make_short4((short)(q.x - X), (short)(q.y - Y), (short)(q.z - X), (short)(q.w - Y));
      else ((int4*)eb)[k] = q;
      const uint64_t m = rmask[x.edge_begin + k];
      if (by) mb[k] = (unsigned char)m; else ((uint64_t*)mb)[k] = m;
    }
  }
}

int bits_for(int64_t v) {  // bits to hold values 0..v
  int b = 1;
  while (b < 63 && (v >> b) != 0) ++b;
  return b;
}

// Build temporaries: stream-ordered allocations from the device's memory pool (kept by the pool
// between builds, keep_pool_memory), freed on the build stream.
struct DevBufs {
  std::vector<void*> ptrs;
  cudaStream_t st;
  explicit DevBufs(cudaStream_t s) : st(s) {}
  ~DevBufs() { for (void* p : ptrs) cudaFreeAsync(p, st); }
  template <class T> cudaError_t alloc(T** p, size_t count) {
    cudaError_t e = cudaMallocAsync((void**)p, std::max<size_t>(count, 1) * sizeof(T), st);
    if (e == cudaSuccess) ptrs.push_back(*p); else *p = nullptr;
    return e;
  }
  void release(void* p) {
    auto it = std::find(ptrs.begin(), ptrs.end(), p);
    if (it != ptrs.end()) { cudaFreeAsync(p, st); ptrs.erase(it); }
  }
};

int grid_for(int64_t n) {
  int64_t g = (n + kBT - 1) / kBT;
  int64_t cap = (int64_t)device_sm_count() * 8;
  return (int)imax64(1, std::min(g, cap));
}

template <class F>
cudaError_t cub_call(DevBufs& bufs, F f) {
  size_t tmp = 0;
  cudaError_t e = f(nullptr, tmp);
  if (e != cudaSuccess) return e;
  void* t = nullptr;
  e = bufs.alloc((char**)&t, tmp);
  if (e != cudaSuccess) return e;
  e = f(t, tmp);
  count_launch();
  return e;
}

}  // namespace

// One builder for both canvas kinds (canvas arrays come from the device's stream-ordered pool,
// so repeated builds -- e.g. the polygon join's two canvases per call -- reuse memory): the front end (K-B0/K-B1 for polygon edges, K-D0/K-D1 for
// disks) produces primitives, boundary fragments and fill events; everything after is shared.
int tile_log2_for(int64_t W0, int64_t H0, int32_t P) {
  // coarse tiles: the shared-memory level holds at most kMaxTiles uint16 entries (<= 160 KB),
  // including one sentinel column and row of always-empty tiles (the probe clamps tile
  // coordinates into them instead of testing the extent); tile side 2^b pixels, s + b <= 30.
  // The probe's COUNT histogram ((P+1) uint32) shares the ~196 KB budget with the tiles.
  const int64_t hist1 = ((int64_t)P + 1) * 4, kSoft = 196 * 1024;
  const int64_t kMaxTiles = hist1 <= kSoft - 8192 ? std::min<int64_t>(81920, std::max<int64_t>(4096, (kSoft - hist1) / 2))
                                                  : 81920;
  int b = 0;
  while ((((W0 + (1 << b) - 1) >> b) + 1) * (((H0 + (1 << b) - 1) >> b) + 1) > kMaxTiles) ++b;
  return b;
}

static int build_any(int kind, const int32_t* ring_xy, const int64_t* ring_off, const int64_t* poly_ring_off,
                     const int32_t* center_xy, const int64_t* r2, int32_t P, const spade_canvas_params* prm,
                     cudaStream_t st, spade_canvas** out, const GridSpec* grid = nullptr) {
  *out = nullptr;
  const char* fn = kind == kDisks ? "spade_build_disk_canvas" : "spade_build_canvas";
  if (P < 0 || (kind == kPolygons && P > 0 && (!ring_off || !poly_ring_off)) || (kind == kDisks && P > 0 && (!center_xy || !r2)))
    return set_error(SPADE_ERR_INVALID_ARG, "%s: bad arguments", fn);
  if (P > (1 << 30)) return set_error(SPADE_ERR_INVALID_ARG, "%s: too many primitives", fn);
  int max_dim = 4096, forced_s = -1;
  if (prm) {
    if (prm->max_dim < 0 || prm->log2_pixel < -1 || prm->log2_pixel > 30)
      return set_error(SPADE_ERR_INVALID_ARG, "%s: bad canvas params", fn);
    if (prm->max_dim > 0) max_dim = prm->max_dim;
    forced_s = prm->log2_pixel;
  }
  if (max_dim < 1 || max_dim > 65536) return set_error(SPADE_ERR_INVALID_ARG, "max_dim out of [1, 65536]");

  cudaError_t ce;
  int64_t V = 0, R = 0;        // V = number of primitives (polygon edges / disks)
  if (kind == kPolygons) {
    // --- offsets to the host for validation (R+1 and P+1 int64s) ---
    std::vector<int64_t> h_pro(P + 1, 0);
    if (P > 0 && (ce = cudaMemcpyAsync(h_pro.data(), poly_ring_off, sizeof(int64_t) * (P + 1), cudaMemcpyDeviceToHost, st)) != cudaSuccess)
      return check_cuda(ce, "copy poly_ring_off");
    if ((ce = cudaStreamSynchronize(st)) != cudaSuccess) return check_cuda(ce, "sync");
    R = h_pro[P];
    if (h_pro[0] != 0 || R < 0) return set_error(SPADE_ERR_INVALID_ARG, "poly_ring_off must start at 0");
    for (int32_t p = 0; p < P; ++p)
      if (h_pro[p + 1] < h_pro[p]) return set_error(SPADE_ERR_INVALID_ARG, "poly_ring_off not non-decreasing at %d", p);
    std::vector<int64_t> h_ro(R + 1, 0);
    if (R > 0) {
      if ((ce = cudaMemcpyAsync(h_ro.data(), ring_off, sizeof(int64_t) * (R + 1), cudaMemcpyDeviceToHost, st)) != cudaSuccess)
        return check_cuda(ce, "copy ring_off");
      if ((ce = cudaStreamSynchronize(st)) != cudaSuccess) return check_cuda(ce, "sync");
    }
    V = h_ro[R];
    if (h_ro[0] != 0 || V < 0) return set_error(SPADE_ERR_INVALID_ARG, "ring_off must start at 0");
    for (int64_t r = 0; r < R; ++r)
      if (h_ro[r + 1] < h_ro[r]) return set_error(SPADE_ERR_INVALID_ARG, "ring_off not non-decreasing at %lld", (long long)r);
    if (V > 0 && !ring_xy) return set_error(SPADE_ERR_INVALID_ARG, "ring_xy is NULL");
    if (V >= (1ll << 31)) return set_error(SPADE_ERR_INVALID_ARG, "too many vertices");
  } else {
    V = P;
  }

  spade_canvas* c = new spade_canvas();
  cudaGetDevice(&c->device);
  c->d.num_polys = P;
  c->d.kind = kind;
  auto fail = [&](int code) { spade_canvas_free(c); return code; };
  if (V == 0) {  // no primitives: every point is outside everything
    c->empty = true;
    *out = c;
    return SPADE_OK;
  }
#define TRYF(call, what) do { cudaError_t _e = (call); if (_e != cudaSuccess) return fail(_e == cudaErrorMemoryAllocation ? set_error(SPADE_ERR_OOM, "build: %s: out of device memory", what) : check_cuda(_e, what)); } while (0)
#define ALLOC(ptr, n, what) TRYF(tmp.alloc(&ptr, (size_t)(n)), what)
#define LAUNCH(kern, n, ...) do { kern<<<grid_for(n), kBT, 0, st>>>(__VA_ARGS__); count_launch(); TRYF(cudaGetLastError(), #kern); } while (0)

  keep_pool_memory();
  StageTimer stages(st);
  stages.mark();                                   // K-B0
  DevBufs tmp(st);
  int4* seg; int32_t* epoly; int* ext; int* bad;
  ALLOC(seg, V, "edges"); ALLOC(epoly, V, "edges"); ALLOC(ext, 4, "ext"); ALLOC(bad, 1, "flag");
  int h_ext0[4] = {INT_MAX, INT_MAX, INT_MIN, INT_MIN};
  TRYF(cudaMemcpyAsync(ext, h_ext0, sizeof(h_ext0), cudaMemcpyHostToDevice, st), "ext init");
  TRYF(cudaMemsetAsync(bad, 0, sizeof(int), st), "memset");
  if (kind == kPolygons) LAUNCH(k_edges, V, (const int2*)ring_xy, ring_off, R, poly_ring_off, P, V, seg, epoly, ext, bad);
  else LAUNCH(k_disks, V, (const int2*)center_xy, r2, P, seg, epoly, ext, bad);
  int h_ext[4], h_bad = 0;
  TRYF(cudaMemcpyAsync(h_ext, ext, sizeof(h_ext), cudaMemcpyDeviceToHost, st), "ext");
  TRYF(cudaMemcpyAsync(&h_bad, bad, sizeof(int), cudaMemcpyDeviceToHost, st), "bad");
  TRYF(cudaStreamSynchronize(st), "sync edges");
  if (kind == kPolygons && h_bad) return fail(set_error(SPADE_ERR_COORD_RANGE, "a polygon vertex lies outside [-2^30, 2^30)"));
  if (kind == kDisks && h_bad == 1) return fail(set_error(SPADE_ERR_INVALID_ARG, "a squared radius lies outside [0, 2^62)"));
  if (kind == kDisks && h_bad) return fail(set_error(SPADE_ERR_COORD_RANGE, "a disk reaches outside [-2^30, 2^30)"));

  // --- canvas geometry (reading C5) ---
  if (grid && (h_ext[0] < grid->minx || h_ext[1] < grid->miny || h_ext[2] > grid->maxx || h_ext[3] > grid->maxy))
    return fail(set_error(SPADE_ERR_INTERNAL, "%s: forced grid does not contain the extent", fn));
  if (grid) { h_ext[0] = grid->minx; h_ext[1] = grid->miny; h_ext[2] = grid->maxx; h_ext[3] = grid->maxy; }
  int64_t ew = (int64_t)h_ext[2] - h_ext[0], eh = (int64_t)h_ext[3] - h_ext[1];
  int s = grid ? grid->s : forced_s;
  if (s < 0) {
    s = 0;
    while (std::max((ew >> s) + 1, (eh >> s) + 1) > max_dim) ++s;
  }
  s = std::min(s, 29);
  Geo g;
  g.minx = h_ext[0]; g.miny = h_ext[1]; g.s = s; g.S = 1ll << s;
  const int64_t W0 = (ew >> s) + 1, H0 = (eh >> s) + 1;
  const int b = grid ? grid->b : tile_log2_for(W0, H0, P);
  if (s + b > 30) return fail(set_error(SPADE_ERR_INVALID_ARG, "canvas tiles too coarse (s=%d, b=%d)", s, b));
  const int Wc = (int)((W0 + (1 << b) - 1) >> b), Hc = (int)((H0 + (1 << b) - 1) >> b);
  // the canvas itself is padded to whole tiles: pixels beyond the extent are ordinary pixels
  // (no edge touches them, no crossing lies right of their corner, so they come out empty)
  const int64_t W64 = (int64_t)Wc << b, H64 = (int64_t)Hc << b;
  if (W64 * H64 > (1ll << 31) - 4) return fail(set_error(SPADE_ERR_INVALID_ARG, "canvas too large (%lld x %lld)", (long long)W64, (long long)H64));
  g.W = (int)W64; g.H = (int)H64;
  const int64_t WH = (int64_t)g.W * g.H;

  // --- K-B1 counts, scans, emit ---
  stages.mark();
  int64_t *nfrag, *nev, *frag_off, *ev_off;
  ALLOC(nfrag, V, "counts"); ALLOC(nev, V, "counts"); ALLOC(frag_off, V + 1, "counts"); ALLOC(ev_off, V + 1, "counts");
  if (kind == kPolygons) LAUNCH(k_count, V, seg, V, g, nfrag, nev);
  else LAUNCH(k_dcount, V, seg, V, g, nfrag, nev);
  for (auto pr : {std::make_pair(nfrag, frag_off), std::make_pair(nev, ev_off)}) {
    int64_t* in = pr.first; int64_t* o = pr.second;
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::InclusiveSum(t, sz, in, o + 1, V, st); }), "scan counts");
    TRYF(cudaMemsetAsync(o, 0, sizeof(int64_t), st), "memset");
  }
  int64_t F = 0, NE = 0;
  TRYF(cudaMemcpyAsync(&F, frag_off + V, 8, cudaMemcpyDeviceToHost, st), "F");
  TRYF(cudaMemcpyAsync(&NE, ev_off + V, 8, cudaMemcpyDeviceToHost, st), "NE");
  TRYF(cudaStreamSynchronize(st), "sync counts");
  tmp.release(nfrag); tmp.release(nev);

  const int pbits = bits_for(std::max<int64_t>(P - 1, 1)), kbits = bits_for(2 * (int64_t)g.W), jbits = bits_for(g.H - 1);
  if (pbits + kbits + jbits > 64) return fail(set_error(SPADE_ERR_INVALID_ARG, "canvas/polygon count too large for event keys"));

  Frag* frags; int64_t* frag_w; uint64_t* ev;
  ALLOC(frags, F, "fragments"); ALLOC(frag_w, F + 1, "fragments"); ALLOC(ev, NE, "events");
  if (kind == kPolygons) LAUNCH(k_emit, V, seg, epoly, V, g, frag_off, ev_off, frags, frag_w, ev, pbits, kbits);
  else LAUNCH(k_demit, V, seg, V, g, frag_off, ev_off, frags, frag_w, ev, pbits, kbits);

  // --- K-B2 boundary pixels, ids, pixel-local edge lists ---
  stages.mark();
  int32_t *bflag, *bscan;
  ALLOC(bflag, WH, "boundary flags"); ALLOC(bscan, WH, "boundary ids");
  TRYF(cudaMemsetAsync(bflag, 0, sizeof(int32_t) * WH, st), "memset");
  if (F > 0) LAUNCH(k_mark, F, frags, F, g.W, bflag);
  TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::InclusiveSum(t, sz, bflag, bscan, WH, st); }), "scan boundary");
  int64_t* lw_off;
  ALLOC(lw_off, F + 1, "local offsets");
  TRYF(cudaMemsetAsync(lw_off, 0, 8, st), "memset");
  if (F > 0)
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::InclusiveSum(t, sz, frag_w, lw_off + 1, F, st); }), "scan local");
  int32_t NB32 = 0; int64_t L = 0;
  TRYF(cudaMemcpyAsync(&NB32, bscan + WH - 1, 4, cudaMemcpyDeviceToHost, st), "NB");
  TRYF(cudaMemcpyAsync(&L, lw_off + F, 8, cudaMemcpyDeviceToHost, st), "L");
  TRYF(cudaStreamSynchronize(st), "sync boundary");
  const int64_t NB = NB32;
  tmp.release(frag_w);
  int64_t *pix_of, *le_beg; int32_t* le_cnt;
  ALLOC(pix_of, NB, "pixel ids"); ALLOC(le_beg, NB + 1, "local edges"); ALLOC(le_cnt, NB, "local edges");
  if (NB > 0) LAUNCH(k_bids, WH, bflag, bscan, WH, pix_of);
  uint64_t *lk, *lk2; int32_t *lv, *lv2;
  ALLOC(lk, L, "local edges"); ALLOC(lk2, L, "local edges"); ALLOC(lv, L, "local edges"); ALLOC(lv2, L, "local edges");
  TRYF(cudaMemsetAsync(le_cnt, 0, sizeof(int32_t) * std::max<int64_t>(NB, 1), st), "memset");
  if (F > 0) LAUNCH(k_local, F, frags, F, g.W, lw_off, epoly, bscan, lk, lv, le_cnt);
  const int bbits = bits_for(std::max<int64_t>(NB - 1, 1));
  if (L > 0)
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceRadixSort::SortPairs(t, sz, lk, lk2, lv, lv2, L, 0, 32 + bbits, st); }), "sort local edges");
  if (NB > 0)
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::ExclusiveSum(t, sz, le_cnt, le_beg, NB, st); }), "scan local edges");
  // distinct polygons per boundary pixel, local indices, de-duplicated edges with toggle masks
  int32_t *ph, *pg, *pbeg, *pcnt, *li, *tix, *tix2, *mcnt;
  int64_t* mbeg;
  uint64_t* key2s;
  ALLOC(ph, L, "dedup"); ALLOC(pg, L, "dedup"); ALLOC(pbeg, NB, "dedup"); ALLOC(pcnt, NB, "dedup");
  ALLOC(li, L, "dedup"); ALLOC(tix, L, "dedup"); ALLOC(tix2, L, "dedup"); ALLOC(key2s, L, "dedup");
  ALLOC(mcnt, NB, "dedup"); ALLOC(mbeg, NB + 1, "dedup");
  int32_t* mkeep; int64_t* mkpos;
  ALLOC(mkeep, L, "dedup"); ALLOC(mkpos, L, "dedup");
  int32_t D32 = 0;
  if (L > 0) {
    LAUNCH(k_polyhead, L, lk2, L, ph);
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::InclusiveSum(t, sz, ph, pg, L, st); }), "scan polys");
    TRYF(cudaMemcpyAsync(&D32, pg + L - 1, 4, cudaMemcpyDeviceToHost, st), "D");
    TRYF(cudaStreamSynchronize(st), "sync polys");
  }
  int32_t* rec_polys;
  ALLOC(rec_polys, D32, "record polygon lists");
  if (L > 0) LAUNCH(k_recpolys, L, lk2, L, ph, pg, rec_polys);
  if (NB > 0) LAUNCH(k_polyrange, NB, NB, le_beg, le_cnt, pg, pbeg, pcnt);
  int64_t LM = 0;
  TRYF(cudaMemsetAsync(mcnt, 0, sizeof(int32_t) * std::max<int64_t>(NB, 1), st), "memset");
  if (L > 0) {
    LAUNCH(k_segkey, L, lk2, lv2, L, seg, pg, pbeg, lk, li);            // lk reused for (bid, hash) keys
    LAUNCH(k_iota, L, tix, L);
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceRadixSort::SortPairs(t, sz, lk, key2s, tix, tix2, L, 0, 32 + bbits, st); }), "sort segments");
    LAUNCH(k_merge<0>, L, key2s, tix2, L, lv2, li, seg, pcnt, le_beg, mcnt, nullptr, mkeep, nullptr, nullptr, nullptr, kind);
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::ExclusiveSum(t, sz, mkeep, mkpos, L, st); }), "scan kept");
  }
  if (NB > 0) {
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::ExclusiveSum(t, sz, mcnt, mbeg, NB, st); }), "scan merged");
    int64_t lb = 0; int32_t lc = 0;
    TRYF(cudaMemcpyAsync(&lb, mbeg + NB - 1, 8, cudaMemcpyDeviceToHost, st), "LM");
    TRYF(cudaMemcpyAsync(&lc, mcnt + NB - 1, 4, cudaMemcpyDeviceToHost, st), "LM");
    TRYF(cudaStreamSynchronize(st), "sync merged");
    LM = lb + lc;
  }
  int4* run_seg; uint64_t* run_mask;
  ALLOC(run_seg, LM, "local edge arrays"); ALLOC(run_mask, LM, "local edge arrays");
  if (L > 0) LAUNCH(k_merge<1>, L, key2s, tix2, L, lv2, li, seg, pcnt, le_beg, mcnt, mbeg, mkeep, mkpos, run_seg, run_mask, kind);
  tmp.release(lk); tmp.release(lk2); tmp.release(lv); tmp.release(lv2); tmp.release(frags); tmp.release(lw_off);
  tmp.release(ph); tmp.release(pg); tmp.release(li); tmp.release(tix); tmp.release(tix2); tmp.release(key2s);

  // --- K-B3 corner owner sets ---
  stages.mark();
  uint64_t* ev2;
  ALLOC(ev2, NE, "events");
  if (NE > 0)
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceRadixSort::SortKeys(t, sz, ev, ev2, NE, 0, jbits + pbits + kbits, st); }), "sort events");
  tmp.release(ev);
  int32_t* corner;
  ALLOC(corner, WH, "corner sets");
  unsigned long long *multi = nullptr, *nmulti;
  int64_t multi_cap = 1 << 20;
  ALLOC(nmulti, 1, "multi");
  unsigned long long h_nmulti = 0;
  for (int attempt = 0; attempt < 2; ++attempt) {
    ALLOC(multi, multi_cap, "multi list");
    TRYF(cudaMemsetAsync(corner, 0xff, sizeof(int32_t) * WH, st), "memset");   // kEmpty
    TRYF(cudaMemsetAsync(nmulti, 0, 8, st), "memset");
    TRYF(cudaMemsetAsync(bad, 0, 4, st), "memset");
    if (NE > 0) LAUNCH(k_fill, (NE + 1) / 2, ev2, NE, g.W, pbits, kbits, corner, multi, nmulti, multi_cap, bad);
    TRYF(cudaMemcpyAsync(&h_nmulti, nmulti, 8, cudaMemcpyDeviceToHost, st), "nmulti");
    TRYF(cudaMemcpyAsync(&h_bad, bad, 4, cudaMemcpyDeviceToHost, st), "bad");
    TRYF(cudaStreamSynchronize(st), "sync fill");
    if (h_bad) return fail(set_error(SPADE_ERR_INTERNAL, "scanline events do not pair up (flag %d)", h_bad));
    if ((int64_t)h_nmulti <= multi_cap) break;
    tmp.release(multi);
    multi_cap = (int64_t)h_nmulti;
  }
  tmp.release(ev2);
  const int64_t M = (int64_t)h_nmulti;
  int64_t NG = 0;
  int32_t* csets = nullptr; int2* crng = nullptr;
  if (M > 0) {
    unsigned long long* m2; int32_t* heads;
    ALLOC(m2, M, "multi sort"); ALLOC(heads, M, "multi sort");
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceRadixSort::SortKeys(t, sz, multi, m2, M, 0, 64, st); }), "sort multi");
    LAUNCH(k_multi_heads, M, m2, M, heads);
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::InclusiveSum(t, sz, heads, heads, M, st); }), "scan multi");
    int32_t ng32 = 0;
    TRYF(cudaMemcpyAsync(&ng32, heads + M - 1, 4, cudaMemcpyDeviceToHost, st), "NG");
    TRYF(cudaStreamSynchronize(st), "sync multi");
    NG = ng32;
    ALLOC(csets, M, "corner sets"); ALLOC(crng, NG, "corner sets");
    LAUNCH(k_multi_sets, M, m2, M, heads, csets, crng, corner);
  }
  tmp.release(multi);

  // --- K-B4 K sets of boundary pixels, records, final canvas ---
  stages.mark();
  int32_t *ksize, *kidx; int64_t* koff;
  ALLOC(ksize, NB, "K sizes"); ALLOC(kidx, NB, "K sizes"); ALLOC(koff, NB + 1, "K offsets");
  int64_t KT = 0; int64_t NK = 0;
  if (NB > 0) {
    LAUNCH(k_kset<0>, NB, NB, pix_of, g, corner, csets, crng, mbeg, mcnt, run_seg, run_mask,
           pbeg, pcnt, rec_polys, ksize, nullptr, nullptr, nullptr, kind);
    thrust::transform_iterator<BigSize, const int32_t*, int64_t, int64_t> it_sz(ksize, BigSize());
    thrust::transform_iterator<BigFlag, const int32_t*, int32_t, int32_t> it_b(ksize, BigFlag());
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::ExclusiveSum(t, sz, it_sz, koff, NB, st); }), "scan K");
    TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::ExclusiveSum(t, sz, it_b, kidx, NB, st); }), "scan K idx");
    int64_t last_off = 0; int32_t last_sz = 0, last_idx = 0;
    TRYF(cudaMemcpyAsync(&last_off, koff + NB - 1, 8, cudaMemcpyDeviceToHost, st), "K");
    TRYF(cudaMemcpyAsync(&last_sz, ksize + NB - 1, 4, cudaMemcpyDeviceToHost, st), "K");
    TRYF(cudaMemcpyAsync(&last_idx, kidx + NB - 1, 4, cudaMemcpyDeviceToHost, st), "K");
    TRYF(cudaStreamSynchronize(st), "sync K");
    KT = last_off + (last_sz >= 2 ? last_sz : 0);
    NK = last_idx + (last_sz >= 2 ? 1 : 0);
  }
  // final set storage: [corner owner sets (M entries, NG ranges)] ++ [K sets with |K| >= 2]
  if (cudaMallocAsync((void**)&c->sets, sizeof(int32_t) * std::max<int64_t>(M + KT, 1), st) != cudaSuccess ||
      cudaMallocAsync((void**)&c->set_rng, sizeof(int2) * std::max<int64_t>(NG + NK, 1), st) != cudaSuccess ||
      cudaMallocAsync((void**)&c->fine, sizeof(int32_t) * WH, st) != cudaSuccess)
    return fail(set_error(SPADE_ERR_OOM, "build: records"));
  RunRec* runs;
  ALLOC(runs, NB + NG, "records");
  if (M > 0) {
    TRYF(cudaMemcpyAsync(c->sets, csets, sizeof(int32_t) * M, cudaMemcpyDeviceToDevice, st), "copy sets");
    TRYF(cudaMemcpyAsync(c->set_rng, crng, sizeof(int2) * NG, cudaMemcpyDeviceToDevice, st), "copy sets");
  }
  if (NB > 0) {
    LAUNCH(k_kset<1>, NB, NB, pix_of, g, corner, csets, crng, mbeg, mcnt, run_seg, run_mask,
           pbeg, pcnt, rec_polys, ksize, koff, c->sets + M, runs, kind);
    LAUNCH(k_kset_rng, NB, NB, ksize, koff, kidx, NG, M, c->set_rng, runs);
  }
  if (NG > 0) LAUNCH(k_multi_recs, NG, NG, NB, runs);

  // --- K-B6 packed records: one contiguous blob (16-B header + data) per record ---
  const int64_t NR = NB + NG;
  int64_t *bsz, *boff;
  uint32_t* bflags;
  ALLOC(bsz, NR, "record blobs"); ALLOC(boff, NR + 1, "record blobs"); ALLOC(bflags, NR, "record blobs");
  LAUNCH(k_blob_size, NR, NR, NB, runs, pix_of, g, run_seg, kind, bsz, bflags);
  TRYF(cudaMemsetAsync(boff, 0, 8, st), "memset");
  TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::InclusiveSum(t, sz, bsz, boff + 1, NR, st); }), "scan blobs");
  int64_t units = 0, multi_unit = 0;
  TRYF(cudaMemcpyAsync(&units, boff + NR, 8, cudaMemcpyDeviceToHost, st), "blob size");
  TRYF(cudaMemcpyAsync(&multi_unit, boff + NB, 8, cudaMemcpyDeviceToHost, st), "blob size");
  TRYF(cudaStreamSynchronize(st), "sync blobs");
  // fine values -2 - offset must stay >= INT32_MIN
  if (units >= (1ll << 31) - 2) return fail(set_error(SPADE_ERR_INVALID_ARG, "boundary index too large (%lld x 16 B)", (long long)units));
  if (cudaMallocAsync((void**)&c->recs, sizeof(Rec) * std::max<int64_t>(NR, 1), st) != cudaSuccess ||
      cudaMallocAsync((void**)&c->blob, 16 * std::max<int64_t>(units, 1), st) != cudaSuccess)
    return fail(set_error(SPADE_ERR_OOM, "build: packed records"));
  c->blob_bytes = 16 * units;
  c->multi_unit = multi_unit;
  TRYF(cudaMemsetAsync(c->blob, 0, 16 * std::max<int64_t>(units, 1), st), "memset blob");   // padding bytes defined
  LAUNCH(k_blob_pack, NR, NR, NB, runs, pix_of, g, run_seg, run_mask, rec_polys, boff, bflags, c->recs, c->blob);
  if (cudaMallocAsync((void**)&c->kbits, sizeof(uint64_t) * std::max<int64_t>(NR, 1), st) != cudaSuccess) return fail(set_error(SPADE_ERR_OOM, "build: K bits"));
  LAUNCH(k_kbits, NR, NR, NB, runs, rec_polys, c->sets, c->set_rng, c->kbits);
  LAUNCH(k_finalize, WH, WH, bflag, bscan, corner, NB, boff, c->fine);

  // --- K-B5 coarse tiles (+ compact fine layout) ---
  stages.mark();
  const int64_t NT = (int64_t)Wc * Hc;
  int32_t *tval, *tmix, *mscan;
  ALLOC(tval, NT, "tiles"); ALLOC(tmix, NT, "tiles"); ALLOC(mscan, NT, "tiles");
  LAUNCH(k_coarse, NT, c->fine, g.W, g.H, b, Wc, Hc, tval, tmix);
  TRYF(cub_call(tmp, [&](void* t, size_t& sz) { return cub::DeviceScan::ExclusiveSum(t, sz, tmix, mscan, NT, st); }), "scan tiles");
  int32_t last_scan = 0, last_mix = 0;
  TRYF(cudaMemcpyAsync(&last_scan, mscan + NT - 1, 4, cudaMemcpyDeviceToHost, st), "mixed");
  TRYF(cudaMemcpyAsync(&last_mix, tmix + NT - 1, 4, cudaMemcpyDeviceToHost, st), "mixed");
  TRYF(cudaStreamSynchronize(st), "sync coarse");
  const int64_t h_mixed = (int64_t)last_scan + last_mix;
  const bool compact = P < (int32_t)kTileMixedCompact - 1 && h_mixed <= 32768 && b <= 8 && !(prm && (prm->flags & SPADE_CANVAS_DENSE));
  const uint32_t owner_lim = compact ? kTileMixedCompact : kTileMixed;     // tile values v+1 below this are uniform
  const int64_t NT1 = (int64_t)(Wc + 1) * (Hc + 1);
  if (cudaMallocAsync((void**)&c->coarse, sizeof(uint16_t) * (NT1 + 16), st) != cudaSuccess)
    return fail(set_error(SPADE_ERR_OOM, "build: coarse"));
  TRYF(cudaMemsetAsync(c->coarse, 0, sizeof(uint16_t) * (NT1 + 16), st), "memset");
  LAUNCH(k_coarse_final, NT1, tval, mscan, Wc, Hc, compact ? 1 : 0, owner_lim, c->coarse);
  if (compact && h_mixed > 0) {
    if (cudaMallocAsync((void**)&c->cfine, sizeof(int32_t) * (h_mixed << (2 * b)), st) != cudaSuccess)
      return fail(set_error(SPADE_ERR_OOM, "build: compact canvas"));
    LAUNCH(k_compact, NT << (2 * b), c->fine, g.W, g.H, b, Wc, tval, mscan, NT, owner_lim, c->cfine);
  }
  const bool f16 = !compact && P < (int32_t)kF16Empty && !(prm && (prm->flags & SPADE_CANVAS_NO_FINE16));
  if (f16) {
    if (cudaMallocAsync((void**)&c->fine16, sizeof(uint16_t) * WH, st) != cudaSuccess) return fail(set_error(SPADE_ERR_OOM, "build: fine16"));
    LAUNCH(k_fine16, WH, c->fine, WH, c->fine16);
  }
  stages.mark();                                   // end of K-B5
  TRYF(cudaStreamSynchronize(st), "sync compact");
  stages.read(c->stage_ms, &c->num_stages);
#undef TRYF
#undef ALLOC
#undef LAUNCH

  c->empty = false;
  c->num_runs = NB;
  c->num_records = NB + NG;
  c->num_run_edges = LM;
  c->num_set_entries = M + KT;
  c->mixed_tile_frac = (double)h_mixed / ((double)Wc * Hc);
  c->num_set_ranges = NG + NK;
  c->cfine_elems = compact ? (h_mixed << (2 * b)) : 0;
  c->coarse_elems = NT1;
  CanvasDev& d = c->d;
  d.minx = (int32_t)g.minx; d.miny = (int32_t)g.miny;
  d.extw = (uint32_t)ew; d.exth = (uint32_t)eh;
  d.s = s; d.W = g.W; d.H = g.H; d.b = b; d.Wc = Wc; d.Hc = Hc;
  d.compact = compact ? 1 : 0;
  d.mix_min = compact ? kTileMixedCompact : kTileMixed;
  d.cfine = c->cfine;
  d.fine = c->fine; d.fine16 = c->fine16; d.f16 = f16 ? 1 : 0; d.coarse = c->coarse; d.recs = c->recs; d.blob = c->blob;
  d.sets = c->sets; d.set_rng = c->set_rng; d.kbits = c->kbits;
  if (cudaMallocAsync((void**)&c->d_dev, sizeof(CanvasDev), st) != cudaSuccess) return fail(set_error(SPADE_ERR_OOM, "build: canvas header"));
  if ((ce = cudaMemcpyAsync(c->d_dev, &d, sizeof(CanvasDev), cudaMemcpyHostToDevice, st)) != cudaSuccess ||
      (ce = cudaStreamSynchronize(st)) != cudaSuccess)
    return fail(check_cuda(ce, "canvas header"));
  *out = c;
  return SPADE_OK;
}

// ---- canvas checksum (replicated-canvas check across ranks) -------------------
// Sum over the 32-bit words w_i of an array of mix(salt, i, w_i) mod 2^64: order-independent, so
// the atomic accumulation is deterministic; any changed word changes the sum (up to 2^-64).
__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__global__ void k_hash(const uint32_t* __restrict__ w, int64_t n, uint64_t salt, unsigned long long* __restrict__ acc) {
  uint64_t h = 0;
  for (int64_t i = blockIdx.x * (int64_t)kBT + threadIdx.x; i < n; i += (int64_t)gridDim.x * kBT)
    h += mix64(salt ^ mix64((uint64_t)i) ^ ((uint64_t)w[i] << 17));
  using BR = cub::BlockReduce<unsigned long long, kBT>;
  __shared__ typename BR::TempStorage tmp;
  const unsigned long long r = BR(tmp).Sum((unsigned long long)h);
  if (threadIdx.x == 0 && r) atomicAdd(acc, r);
}

int canvas_checksum(const spade_canvas* c, uint64_t* out, cudaStream_t st) {
  uint64_t h = mix64(0x5ADEull ^ (uint64_t)c->d.num_polys ^ ((uint64_t)c->d.kind << 40));
  if (!c->empty) {
    const CanvasDev& d = c->d;
    const int64_t hdr[] = {d.minx, d.miny, d.extw, d.exth, d.s, d.W, d.H, d.b, d.Wc, d.Hc, d.compact, d.mix_min, d.f16,
                           c->num_runs, c->num_records, c->num_run_edges, c->num_set_entries, c->num_set_ranges,
                           c->multi_unit};
    for (int64_t v : hdr) h = mix64(h ^ (uint64_t)v);
    unsigned long long* acc = nullptr;
    cudaError_t e = cudaMallocAsync((void**)&acc, sizeof(unsigned long long), st);
    if (e != cudaSuccess) return check_cuda(e, "spade_canvas_checksum");
    e = cudaMemsetAsync(acc, 0, sizeof(unsigned long long), st);
    struct A { const void* p; int64_t words; };
    const A arrs[] = {{c->fine, (int64_t)d.W * d.H}, {c->fine16, c->fine16 ? ((int64_t)d.W * d.H + 1) / 2 : 0},
                      {c->cfine, c->cfine_elems}, {c->coarse, (c->coarse_elems + 1) / 2},
                      {c->recs, c->num_records * (int64_t)(sizeof(Rec) / 4)}, {c->blob, c->blob_bytes / 4},
                      {c->sets, c->num_set_entries}, {c->set_rng, 2 * c->num_set_ranges},
                      {c->kbits, 2 * c->num_records}};
    uint64_t salt = 1;
    for (const A& a : arrs) {
      if (e == cudaSuccess && a.p && a.words > 0) {
        k_hash<<<grid_for(a.words), kBT, 0, st>>>((const uint32_t*)a.p, a.words, mix64(salt), acc);
        count_launch();
        e = cudaGetLastError();
      }
      ++salt;
    }
    unsigned long long r = 0;
    if (e == cudaSuccess) e = cudaMemcpyAsync(&r, acc, sizeof(r), cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    cudaFreeAsync(acc, st);
    if (e != cudaSuccess) return check_cuda(e, "spade_canvas_checksum");
    h = mix64(h ^ (uint64_t)r);
  }
  *out = h;
  return SPADE_OK;
}

int build_canvas_on_grid(const int32_t* ring_xy, const int64_t* ring_off, const int64_t* poly_ring_off, int32_t P,
                         const GridSpec& grid, cudaStream_t st, spade_canvas** out) {
  spade_canvas_params prm{grid.s, 0, SPADE_CANVAS_DENSE | SPADE_CANVAS_NO_FINE16};
  return build_any(kPolygons, ring_xy, ring_off, poly_ring_off, nullptr, nullptr, P, &prm, st, out, &grid);
}

int build_canvas(const int32_t* ring_xy, const int64_t* ring_off, const int64_t* poly_ring_off, int32_t P,
                 const spade_canvas_params* prm, cudaStream_t st, spade_canvas** out) {
  return build_any(kPolygons, ring_xy, ring_off, poly_ring_off, nullptr, nullptr, P, prm, st, out);
}

int build_disk_canvas(const int32_t* center_xy, const int64_t* r2, int32_t D, const spade_canvas_params* prm,
                      cudaStream_t st, spade_canvas** out) {
  return build_any(kDisks, nullptr, nullptr, nullptr, center_xy, r2, D, prm, st, out);
}

}  // namespace spade
