// polygon_join.cu — spade_join_polygons: the Polygon x Polygon join (Sec. 5.2).
//
// Result: every pair (a, b), a in D1, b in D2, whose CLOSED regions intersect (ST_INTERSECTS,
// P:184; reading C15).  Exactly that set is the union of two parts:
//   (1) boundary contact: some edge of a and some edge of b share a point;
//   (2) containment without contact: the first vertex of some ring of one polygon lies inside
//       the other (if the boundaries do not meet, a whole ring of one lies in the other).
// The paper runs one selection per layer of D1 against D2's canvas and tests boundary
// pixels through the boundary index (polygon-polygon tests become local tests).  Here both
// sets are rasterised on ONE pixel grid (same extent, pixel and tile size), so:
//   (1) an edge contact point lies in a closed pixel touched by both edges, i.e. in a pixel that
//       is a boundary pixel of both canvases, whose records list exactly the edges touching it:
//       k_pp_contacts tests only those local edge pairs (exact closed-segment test in int64);
//   (2) is a point join: the first vertices of D2's rings probed against D1's canvas and those of
//       D1's rings against D2's canvas (the half-open point rule decides them exactly: a vertex
//       on the other polygon's boundary is a contact already found by (1)).
// Pairs are 64-bit keys (a << 32 | b); one radix sort + unique gives the sorted, duplicate-free
// output.  Domain (as the oracle): valid polygons -- rings of >= 3 vertices, no zero-length edge,
// no segment used twice by one polygon.
#include <cub/cub.cuh>
#include <algorithm>
#include <vector>
#include "spade_internal.cuh"

namespace spade {

int launch_pairs(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t base, int64_t* opt, int32_t* opl,
                 int64_t cap, unsigned long long* d_total, cudaStream_t st);

namespace {

constexpr int kPJ = 256;

int pj_grid(int64_t n) {
  return (int)std::max<int64_t>(1, std::min<int64_t>((n + kPJ - 1) / kPJ, (int64_t)device_sm_count() * 8));
}

// extent of a vertex array: ext = {minx, miny, maxx, maxy}
__global__ void k_vert_extent(const int2* __restrict__ xy, int64_t V, int* __restrict__ ext) {
  using BR = cub::BlockReduce<int, kPJ>;
  __shared__ typename BR::TempStorage tmp;
  int mnx = INT_MAX, mny = INT_MAX, mxx = INT_MIN, mxy = INT_MIN;
  for (int64_t k = blockIdx.x * (int64_t)kPJ + threadIdx.x; k < V; k += (int64_t)gridDim.x * kPJ) {
    const int2 v = xy[k];
    mnx = min(mnx, v.x); mny = min(mny, v.y); mxx = max(mxx, v.x); mxy = max(mxy, v.y);
  }
  int r = BR(tmp).Reduce(mnx, cub::Min()); __syncthreads(); if (threadIdx.x == 0) atomicMin(&ext[0], r);
  r = BR(tmp).Reduce(mny, cub::Min()); __syncthreads(); if (threadIdx.x == 0) atomicMin(&ext[1], r);
  r = BR(tmp).Reduce(mxx, cub::Max()); __syncthreads(); if (threadIdx.x == 0) atomicMax(&ext[2], r);
  r = BR(tmp).Reduce(mxy, cub::Max()); if (threadIdx.x == 0) atomicMax(&ext[3], r);
}

// first vertex of every ring (the containment probe points) and the ring's polygon
__global__ void k_ring_v0(const int2* __restrict__ xy, const int64_t* __restrict__ ring_off, int64_t R,
                          const int64_t* __restrict__ poly_ring_off, int32_t P, int2* __restrict__ v0,
                          int32_t* __restrict__ ring_poly) {
  for (int64_t r = blockIdx.x * (int64_t)kPJ + threadIdx.x; r < R; r += (int64_t)gridDim.x * kPJ) {
    // an empty ring probes a point outside every canvas (INT32_MIN: clamped into the sentinels)
    v0[r] = ring_off[r + 1] > ring_off[r] ? xy[ring_off[r]] : make_int2(INT32_MIN, INT32_MIN);
    int64_t lo = 0, hi = (int64_t)P + 1;          // polygon p: poly_ring_off[p] <= r < poly_ring_off[p + 1]
    while (hi - lo > 1) { const int64_t mid = (lo + hi) >> 1; if (poly_ring_off[mid] <= r) lo = mid; else hi = mid; }
    ring_poly[r] = (int32_t)lo;
  }
}

// sign of (q - p) x (r - p); coordinates in [-2^30, 2^30): differences < 2^31, products < 2^62
__device__ __forceinline__ int orient(int px, int py, int qx, int qy, int rx, int ry) {
  const long long v = (long long)(qx - px) * (ry - py) - (long long)(qy - py) * (rx - px);
  return (v > 0) - (v < 0);
}
__device__ __forceinline__ bool within(int px, int py, int qx, int qy, int rx, int ry) {
  return rx >= min(px, qx) && rx <= max(px, qx) && ry >= min(py, qy) && ry <= max(py, qy);
}
// closed segments a and b share a point (straddle both ways, or a collinear endpoint within)
__device__ __forceinline__ bool seg_touch(int4 a, int4 b) {
  const int d1 = orient(b.x, b.y, b.z, b.w, a.x, a.y), d2 = orient(b.x, b.y, b.z, b.w, a.z, a.w);
  const int d3 = orient(a.x, a.y, a.z, a.w, b.x, b.y), d4 = orient(a.x, a.y, a.z, a.w, b.z, b.w);
  if (d1 * d2 < 0 && d3 * d4 < 0) return true;
  return (d1 == 0 && within(b.x, b.y, b.z, b.w, a.x, a.y)) || (d2 == 0 && within(b.x, b.y, b.z, b.w, a.z, a.w)) ||
         (d3 == 0 && within(a.x, a.y, a.z, a.w, b.x, b.y)) || (d4 == 0 && within(a.x, a.y, a.z, a.w, b.z, b.w));
}

// a boundary record's edges in absolute coordinates (spade_internal.cuh "Packed records")
struct RecEdges {
  const unsigned char* prims;
  const unsigned char* masks;
  const int32_t* polys;
  int ne, pc, X, Y;
  bool sh, by;
  __device__ __forceinline__ RecEdges(const CanvasDev& cv, uint32_t u, int X_, int Y_) : X(X_), Y(Y_) {
    const uint4 h = __ldg(cv.blob + u);
    ne = (int)h.y;
    pc = (int)(h.z & kRecPcnt);
    sh = h.z & kRecShort;
    by = h.z & kRecByte;
    polys = (const int32_t*)(cv.blob + u + 1);
    prims = (const unsigned char*)polys + ((pc * 4 + 15) & ~15);
    masks = prims + (size_t)ne * (sh ? 8 : 16);
  }
  __device__ __forceinline__ int4 edge(int k) const {
    if (sh) {
      const short4 v = __ldg((const short4*)prims + k);
      return make_int4(X + v.x, Y + v.y, X + v.z, Y + v.w);
    }
    return __ldg((const int4*)prims + k);
  }
  // polygons using edge k: a bit mask of local indices (pc <= 64), else one local index
  __device__ __forceinline__ uint64_t mask(int k) const {
    return by ? (uint64_t)__ldg(masks + k) : __ldg((const uint64_t*)masks + k);
  }
};

// (1) boundary contacts: pixels that are boundary pixels of both canvases, every pair of their
// local edges; a touching pair emits (polygon of a's edge, polygon of b's edge) for every polygon
// using each edge.  Keys past `cap` are counted, not stored.
__global__ void k_pp_contacts(const CanvasDev A, const CanvasDev B, int64_t WH, unsigned long long* __restrict__ keys,
                              unsigned long long cap, unsigned long long* __restrict__ cnt) {
  for (int64_t p = blockIdx.x * (int64_t)kPJ + threadIdx.x; p < WH; p += (int64_t)gridDim.x * kPJ) {
    const int32_t va = __ldg(A.fine + p), vb = __ldg(B.fine + p);
    if (va > -2 || vb > -2) continue;
    const int X = A.minx + (int)(((uint32_t)(p % (uint32_t)A.W)) << A.s);
    const int Y = A.miny + (int)(((uint32_t)(p / (uint32_t)A.W)) << A.s);
    const RecEdges ra(A, (uint32_t)(-2 - va), X, Y), rb(B, (uint32_t)(-2 - vb), X, Y);
    for (int i = 0; i < ra.ne; ++i) {
      const int4 ea = ra.edge(i);
      for (int j = 0; j < rb.ne; ++j) {
        if (!seg_touch(ea, rb.edge(j))) continue;
        const uint64_t ma = ra.mask(i), mb = rb.mask(j);
        const bool bigA = ra.pc > kMaskPolys, bigB = rb.pc > kMaskPolys;
        for (uint64_t xa = bigA ? 1 : ma; xa; xa &= xa - 1) {
          const int32_t pa = __ldg(ra.polys + (bigA ? (int)ma : __ffsll((long long)xa) - 1));
          for (uint64_t xb = bigB ? 1 : mb; xb; xb &= xb - 1) {
            const int32_t pb = __ldg(rb.polys + (bigB ? (int)mb : __ffsll((long long)xb) - 1));
            const unsigned long long q = atomicAdd(cnt, 1ull);
            if (q < cap) keys[q] = ((unsigned long long)(uint32_t)pa << 32) | (uint32_t)pb;
          }
        }
      }
    }
  }
}

// (2) containment pairs from the point join of ring first vertices: point id = ring index
__global__ void k_ring_keys(const int64_t* __restrict__ ring_ids, const int32_t* __restrict__ hit_poly, int64_t n,
                            const int32_t* __restrict__ ring_poly, int vertex_side_is_b,
                            unsigned long long* __restrict__ keys) {
  for (int64_t t = blockIdx.x * (int64_t)kPJ + threadIdx.x; t < n; t += (int64_t)gridDim.x * kPJ) {
    const uint32_t q = (uint32_t)ring_poly[ring_ids[t]], h = (uint32_t)hit_poly[t];
    keys[t] = vertex_side_is_b ? ((unsigned long long)h << 32) | q : ((unsigned long long)q << 32) | h;
  }
}

__global__ void k_split_keys(const unsigned long long* __restrict__ keys, int64_t n, int32_t* __restrict__ a,
                             int32_t* __restrict__ b) {
  for (int64_t t = blockIdx.x * (int64_t)kPJ + threadIdx.x; t < n; t += (int64_t)gridDim.x * kPJ) {
    const unsigned long long k = keys[t];
    a[t] = (int32_t)(k >> 32);
    b[t] = (int32_t)(uint32_t)k;
  }
}

struct PoolBufs {                                   // stream-ordered temporaries
  std::vector<void*> ptrs;
  cudaStream_t st;
  explicit PoolBufs(cudaStream_t s) : st(s) {}
  ~PoolBufs() { for (void* p : ptrs) cudaFreeAsync(p, st); }
  template <class T> cudaError_t alloc(T** p, size_t n) {
    cudaError_t e = cudaMallocAsync((void**)p, std::max<size_t>(n, 1) * sizeof(T), st);
    if (e == cudaSuccess) ptrs.push_back(*p); else *p = nullptr;
    return e;
  }
};

struct CanvasGuard {
  spade_canvas* c = nullptr;
  ~CanvasGuard() { if (c) spade_canvas_free(c); }
};

int host_counts(const int64_t* poly_ring_off, const int64_t* ring_off, int32_t P, int64_t& R, int64_t& V, cudaStream_t st) {
  R = V = 0;
  if (P <= 0) return SPADE_OK;
  cudaError_t e = cudaMemcpyAsync(&R, poly_ring_off + P, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e == cudaSuccess && R > 0) e = cudaMemcpyAsync(&V, ring_off + R, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  return check_cuda(e, "spade_join_polygons: offsets");
}

}  // namespace

int join_polygons(const int32_t* xy1, const int64_t* ro1, const int64_t* pro1, int32_t n1, const int32_t* xy2,
                  const int64_t* ro2, const int64_t* pro2, int32_t n2, const spade_canvas_params* prm, int32_t* out_a,
                  int32_t* out_b, int64_t capacity, int64_t* n_out, cudaStream_t st) {
  const char* fn = "spade_join_polygons";
  *n_out = 0;
  if (n1 < 0 || n2 < 0 || capacity < 0) return set_error(SPADE_ERR_INVALID_ARG, "%s: bad arguments", fn);
  if ((n1 > 0 && (!ro1 || !pro1)) || (n2 > 0 && (!ro2 || !pro2)) || (capacity > 0 && (!out_a || !out_b)))
    return set_error(SPADE_ERR_INVALID_ARG, "%s: NULL array", fn);
  int64_t R1, V1, R2, V2;
  int rc = host_counts(pro1, ro1, n1, R1, V1, st);
  if (rc == SPADE_OK) rc = host_counts(pro2, ro2, n2, R2, V2, st);
  if (rc != SPADE_OK) return rc;
  if (V1 == 0 || V2 == 0) return SPADE_OK;                    // a set without vertices meets nothing
  if ((V1 > 0 && !xy1) || (V2 > 0 && !xy2)) return set_error(SPADE_ERR_INVALID_ARG, "%s: NULL vertices", fn);
  keep_pool_memory();
  PoolBufs tmp(st);
#define PJ_TRY(call, what) do { cudaError_t e_ = (call); if (e_ != cudaSuccess) return check_cuda(e_, what); } while (0)
  // one grid for both sets: the union extent, the pixel size max_dim picks for it, one tile size
  int* ext;
  PJ_TRY(tmp.alloc(&ext, 4), fn);
  const int ext0[4] = {INT_MAX, INT_MAX, INT_MIN, INT_MIN};
  PJ_TRY(cudaMemcpyAsync(ext, ext0, sizeof(ext0), cudaMemcpyHostToDevice, st), fn);
  k_vert_extent<<<pj_grid(V1), kPJ, 0, st>>>((const int2*)xy1, V1, ext);
  k_vert_extent<<<pj_grid(V2), kPJ, 0, st>>>((const int2*)xy2, V2, ext);
  count_launch(2);
  int h_ext[4];
  PJ_TRY(cudaMemcpyAsync(h_ext, ext, sizeof(h_ext), cudaMemcpyDeviceToHost, st), fn);
  PJ_TRY(cudaStreamSynchronize(st), fn);
  const int lim = 1 << 30;
  if (h_ext[0] < -lim || h_ext[1] < -lim || h_ext[2] >= lim || h_ext[3] >= lim)
    return set_error(SPADE_ERR_COORD_RANGE, "%s: a polygon vertex lies outside [-2^30, 2^30)", fn);
  int max_dim = prm && prm->max_dim > 0 ? prm->max_dim : 4096;
  if (max_dim > 65536) return set_error(SPADE_ERR_INVALID_ARG, "%s: max_dim out of [1, 65536]", fn);
  const int64_t ew = (int64_t)h_ext[2] - h_ext[0], eh = (int64_t)h_ext[3] - h_ext[1];
  int s = prm && prm->log2_pixel >= 0 ? std::min(prm->log2_pixel, 29) : -1;
  if (s < 0) { s = 0; while (std::max((ew >> s) + 1, (eh >> s) + 1) > max_dim) ++s; }
  const GridSpec grid{h_ext[0], h_ext[1], h_ext[2], h_ext[3], s,
                      tile_log2_for((ew >> s) + 1, (eh >> s) + 1, std::max(n1, n2))};
  CanvasGuard ca, cb;
  rc = build_canvas_on_grid(xy1, ro1, pro1, n1, grid, st, &ca.c);
  if (rc == SPADE_OK) rc = build_canvas_on_grid(xy2, ro2, pro2, n2, grid, st, &cb.c);
  if (rc != SPADE_OK) return rc;
  const CanvasDev& A = ca.c->d;
  const CanvasDev& B = cb.c->d;
  const int64_t WH = (int64_t)A.W * A.H;

  // (1) boundary contacts (counted first if the first guess of the buffer is too small)
  unsigned long long* d_cnt;
  PJ_TRY(tmp.alloc(&d_cnt, 3), fn);
  unsigned long long ccap = (unsigned long long)std::max<int64_t>(1 << 16, 4 * (ca.c->num_run_edges + cb.c->num_run_edges));
  unsigned long long* ckeys = nullptr;
  unsigned long long h_cnt = 0;
  for (int attempt = 0; attempt < 2; ++attempt) {
    PJ_TRY(tmp.alloc(&ckeys, ccap), fn);
    PJ_TRY(cudaMemsetAsync(d_cnt, 0, 8, st), fn);
    if (!ca.c->empty && !cb.c->empty) {
      k_pp_contacts<<<pj_grid(WH), kPJ, 0, st>>>(A, B, WH, ckeys, ccap, d_cnt);
      count_launch();
      PJ_TRY(cudaGetLastError(), "k_pp_contacts");
    }
    PJ_TRY(cudaMemcpyAsync(&h_cnt, d_cnt, 8, cudaMemcpyDeviceToHost, st), fn);
    PJ_TRY(cudaStreamSynchronize(st), fn);
    if (h_cnt <= ccap) break;
    ccap = h_cnt;
  }

  // (2) containment: ring first vertices of each set probed against the other set's canvas
  int64_t nv[2] = {0, 0};
  unsigned long long* vkeys[2] = {nullptr, nullptr};
  for (int side = 0; side < 2; ++side) {
    const int64_t R = side == 0 ? R2 : R1;                   // side 0: D2's rings in D1's canvas
    const spade_canvas* cv = side == 0 ? ca.c : cb.c;
    const int2* vxy = (const int2*)(side == 0 ? xy2 : xy1);
    int2* v0; int32_t* rpoly; int64_t* ids; int32_t* hit; unsigned long long* dt;
    PJ_TRY(tmp.alloc(&v0, R), fn); PJ_TRY(tmp.alloc(&rpoly, R), fn); PJ_TRY(tmp.alloc(&dt, 1), fn);
    k_ring_v0<<<pj_grid(R), kPJ, 0, st>>>(vxy, side == 0 ? ro2 : ro1, R, side == 0 ? pro2 : pro1, side == 0 ? n2 : n1, v0, rpoly);
    count_launch();
    int64_t cap = R;
    for (int attempt = 0; attempt < 2; ++attempt) {
      PJ_TRY(tmp.alloc(&ids, cap), fn); PJ_TRY(tmp.alloc(&hit, cap), fn);
      PJ_TRY(cudaMemsetAsync(dt, 0, 8, st), fn);
      rc = launch_pairs(cv, (const int32_t*)v0, R, 0, ids, hit, cap, dt, st);
      if (rc != SPADE_OK) return rc;
      unsigned long long h = 0;
      PJ_TRY(cudaMemcpyAsync(&h, dt, 8, cudaMemcpyDeviceToHost, st), fn);
      PJ_TRY(cudaStreamSynchronize(st), fn);
      nv[side] = (int64_t)h;
      if ((int64_t)h <= cap) break;
      cap = (int64_t)h;
    }
    PJ_TRY(tmp.alloc(&vkeys[side], nv[side]), fn);
    if (nv[side] > 0) {
      k_ring_keys<<<pj_grid(nv[side]), kPJ, 0, st>>>(ids, hit, nv[side], rpoly, side == 0 ? 1 : 0, vkeys[side]);
      count_launch();
    }
  }

  // all candidate keys -> sorted unique pairs
  const int64_t total = (int64_t)h_cnt + nv[0] + nv[1];
  unsigned long long *all, *sorted, *uniq;
  int64_t* d_nu;
  PJ_TRY(tmp.alloc(&all, total), fn); PJ_TRY(tmp.alloc(&sorted, total), fn); PJ_TRY(tmp.alloc(&uniq, total), fn);
  PJ_TRY(tmp.alloc(&d_nu, 1), fn);
  if (h_cnt) PJ_TRY(cudaMemcpyAsync(all, ckeys, 8 * h_cnt, cudaMemcpyDeviceToDevice, st), fn);
  if (nv[0]) PJ_TRY(cudaMemcpyAsync(all + h_cnt, vkeys[0], 8 * nv[0], cudaMemcpyDeviceToDevice, st), fn);
  if (nv[1]) PJ_TRY(cudaMemcpyAsync(all + h_cnt + nv[0], vkeys[1], 8 * nv[1], cudaMemcpyDeviceToDevice, st), fn);
  int64_t nu = 0;
  if (total > 0) {
    int bits = 33;
    while (bits < 64 && ((int64_t)1 << (bits - 32)) < (int64_t)n1) ++bits;
    size_t tb = 0;
    PJ_TRY(cub::DeviceRadixSort::SortKeys(nullptr, tb, all, sorted, total, 0, bits, st), fn);
    void* t1; PJ_TRY(tmp.alloc((char**)&t1, tb), fn);
    PJ_TRY(cub::DeviceRadixSort::SortKeys(t1, tb, all, sorted, total, 0, bits, st), fn);
    size_t tu = 0;
    PJ_TRY(cub::DeviceSelect::Unique(nullptr, tu, sorted, uniq, d_nu, total, st), fn);
    void* t2; PJ_TRY(tmp.alloc((char**)&t2, tu), fn);
    PJ_TRY(cub::DeviceSelect::Unique(t2, tu, sorted, uniq, d_nu, total, st), fn);
    count_launch(2);
    PJ_TRY(cudaMemcpyAsync(&nu, d_nu, 8, cudaMemcpyDeviceToHost, st), fn);
    PJ_TRY(cudaStreamSynchronize(st), fn);
    const int64_t keep = std::min(nu, capacity);
    if (keep > 0) {
      k_split_keys<<<pj_grid(keep), kPJ, 0, st>>>(uniq, keep, out_a, out_b);
      count_launch();
      PJ_TRY(cudaGetLastError(), "k_split_keys");
    }
  }
  PJ_TRY(cudaStreamSynchronize(st), fn);
#undef PJ_TRY
  *n_out = nu;
  if (nu > capacity)
    return set_error(SPADE_ERR_CAPACITY, "%s: %lld pairs exceed capacity %lld", fn, (long long)nu, (long long)capacity);
  return SPADE_OK;
}

}  // namespace spade
