// canvas_build.cu — spade_build_canvas: exact integer rasterisation of polygons into the discrete
// canvas + boundary index (Sec. 4.2 canvas creation P:113-123, Sec. 4.3 boundary index
// P:140-146, Sec. 5.5 boundary-index creation P:268).  Replaces the paper's OpenGL pipeline
// (triangulation P:117, two-pass triangle/line render P:121, conservative rasterisation P:123)
// with data-parallel kernels:
//   K-B1  edge -> (row, pixel-range) fragments of every closed pixel an edge touches; mark them
//   K-B2  maximal runs of boundary pixels per row; run -> edge CSR sorted by polygon
//   K-B3  scanline crossing events at each row's bottom line; per (row, polygon) pairs of events
//         bound interior spans; fill the non-boundary pixels (multi-owner pixels -> records)
//   K-B4  terminal owner set of each run = owner set of the first non-boundary pixel to its right
//   K-B5  coarse tile summary (uniform owner / empty / mixed) for the shared-memory level
// DESIGN.md "Canvas" has the exactness argument for the run-local PIP this enables.
#include <cub/cub.cuh>
#include <vector>
#include <algorithm>
#include "spade_internal.cuh"

namespace spade {

namespace {

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
                        int64_t* __restrict__ nlist, int64_t* __restrict__ nev) {
  for (int64_t k = blockIdx.x * (int64_t)kBT + threadIdx.x; k < E; k += (int64_t)gridDim.x * kBT) {
    int4 e = seg[k];
    int64_t a, b;
    frag_rows(e, g, a, b);
    int64_t nf = b >= a ? b - a + 1 : 0;
    nfrag[k] = nf;
    nlist[k] = (e.y != e.w) ? nf : 0;        // horizontal edges never straddle: not listed
    int64_t c0, c1;
    event_rows(e, g, c0, c1);
    nev[k] = (e.y != e.w && c1 >= c0) ? c1 - c0 + 1 : 0;
  }
}

struct Frag { int32_t j, ilo, ihi, e; };

__global__ void k_emit(const int4* __restrict__ seg, const int32_t* __restrict__ poly, int64_t E, Geo g,
                       const int64_t* __restrict__ frag_off, const int64_t* __restrict__ ev_off,
                       Frag* __restrict__ frags, uint64_t* __restrict__ ev_keys, int pbits, int cbits) {
  for (int64_t k = blockIdx.x * (int64_t)kBT + threadIdx.x; k < E; k += (int64_t)gridDim.x * kBT) {
    int4 e = seg[k];
    int64_t a, b;
    frag_rows(e, g, a, b);
    int64_t o = frag_off[k];
    for (int64_t j = a; j <= b; ++j, ++o) {
      int ilo, ihi;
      frag_cols(e, g, j, ilo, ihi);
      frags[o] = Frag{(int32_t)j, ilo, ihi, (int32_t)k};
    }
    if (e.y == e.w) continue;
    event_rows(e, g, a, b);
    o = ev_off[k];
    int64_t dx = (int64_t)e.z - e.x, dy = (int64_t)e.w - e.y;
    uint64_t pk = (uint64_t)poly[k];
    for (int64_t j = a; j <= b; ++j, ++o) {
      int64_t Y0 = g.miny + j * g.S;
      int64_t xf = e.x + floor_div(dx * (Y0 - e.y), dy);   // floor of the crossing x*
      int64_t c = floor_div(xf - g.minx, g.S);              // pixel column holding x*
      ev_keys[o] = ((uint64_t)j << (pbits + cbits)) | (pk << cbits) | (uint64_t)c;
    }
  }
}

__global__ void k_mark(const Frag* __restrict__ frags, int64_t F, int W, uint8_t* __restrict__ bmap) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < F; t += (int64_t)gridDim.x * kBT) {
    Frag f = frags[t];
    uint8_t* row = bmap + (int64_t)f.j * W;
    for (int i = f.ilo; i <= f.ihi; ++i) row[i] = 1;
  }
}

__global__ void k_run_flags(const uint8_t* __restrict__ bmap, int64_t WH, int W, int32_t* __restrict__ flag) {
  for (int64_t p = blockIdx.x * (int64_t)kBT + threadIdx.x; p < WH; p += (int64_t)gridDim.x * kBT) {
    int i = (int)(p % W);
    flag[p] = (bmap[p] && (i == 0 || !bmap[p - 1])) ? 1 : 0;
  }
}

// after the inclusive scan: run id of boundary pixel p = scan[p] - 1
__global__ void k_run_ids(const uint8_t* __restrict__ bmap, const int32_t* __restrict__ scan, int64_t WH, int W,
                          int32_t* __restrict__ fine, int64_t* __restrict__ run_end) {
  for (int64_t p = blockIdx.x * (int64_t)kBT + threadIdx.x; p < WH; p += (int64_t)gridDim.x * kBT) {
    if (!bmap[p]) { fine[p] = kEmpty; continue; }
    int32_t r = scan[p] - 1;
    fine[p] = -2 - r;
    int i = (int)(p % W);
    if (i == W - 1 || !bmap[p + 1]) run_end[r] = p;
  }
}

__global__ void k_list(const Frag* __restrict__ frags, int64_t F, int W, const int4* __restrict__ seg,
                       const int32_t* __restrict__ poly, const int32_t* __restrict__ scan,
                       const int64_t* __restrict__ frag_off, const int64_t* __restrict__ list_off,
                       uint64_t* __restrict__ keys, int32_t* __restrict__ vals, int32_t* __restrict__ run_cnt) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < F; t += (int64_t)gridDim.x * kBT) {
    Frag f = frags[t];
    int4 e = seg[f.e];
    if (e.y == e.w) continue;
    int32_t run = scan[(int64_t)f.j * W + f.ilo] - 1;   // all of [ilo, ihi] lies in this run
    int64_t pos = list_off[f.e] + (t - frag_off[f.e]);
    keys[pos] = ((uint64_t)(uint32_t)run << 32) | (uint32_t)poly[f.e];
    vals[pos] = f.e;
    atomicAdd(&run_cnt[run], 1);
  }
}

__global__ void k_gather_edges(const int32_t* __restrict__ sorted_e, int64_t L, const int4* __restrict__ seg,
                               const int32_t* __restrict__ poly, int4* __restrict__ run_seg,
                               int32_t* __restrict__ run_poly) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < L; t += (int64_t)gridDim.x * kBT) {
    int32_t e = sorted_e[t];
    run_seg[t] = seg[e];
    run_poly[t] = poly[e];
  }
}

// K-B3 fill: sorted events of one (row, polygon) come in consecutive pairs (every closed ring
// crosses a horizontal line an even number of times); non-boundary pixels strictly between the
// pair's columns have the polygon's parity odd at their lower-left corner.
__global__ void k_fill(const uint64_t* __restrict__ ev, int64_t NE, int W, int pbits, int cbits,
                       const uint8_t* __restrict__ bmap, int32_t* __restrict__ fine,
                       unsigned long long* __restrict__ multi, unsigned long long* __restrict__ nmulti,
                       int64_t multi_cap, int* __restrict__ bad) {
  const uint64_t cmask = (1ull << cbits) - 1, pmask = (1ull << pbits) - 1;
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; 2 * t + 1 < NE + 1; t += (int64_t)gridDim.x * kBT) {
    if (2 * t + 1 >= NE) { atomicOr(bad, 2); break; }
    uint64_t k0 = ev[2 * t], k1 = ev[2 * t + 1];
    if ((k0 >> cbits) != (k1 >> cbits)) { atomicOr(bad, 2); continue; }
    int64_t j = (int64_t)(k0 >> (cbits + pbits));
    int32_t p = (int32_t)((k0 >> cbits) & pmask);
    int ca = (int)(k0 & cmask), cb = (int)(k1 & cmask);
    int64_t rowbase = j * W;
    for (int i = ca + 1; i < cb; ++i) {
      int64_t px = rowbase + i;
      if (bmap[px]) continue;
      int old = atomicCAS(&fine[px], kEmpty, p);
      if (old == kEmpty) continue;
      int prev = atomicExch(&fine[px], kMultiMark);
      unsigned long long q = atomicAdd(nmulti, prev >= 0 ? 2ull : 1ull);
      if ((int64_t)q < multi_cap) multi[q] = ((unsigned long long)px << 32) | (uint32_t)p;
      if (prev >= 0 && (int64_t)q + 1 < multi_cap) multi[q + 1] = ((unsigned long long)px << 32) | (uint32_t)prev;
    }
  }
}

__global__ void k_reset_fill(const uint8_t* __restrict__ bmap, int64_t WH, int32_t* __restrict__ fine) {
  for (int64_t p = blockIdx.x * (int64_t)kBT + threadIdx.x; p < WH; p += (int64_t)gridDim.x * kBT)
    if (!bmap[p]) fine[p] = kEmpty;
}

// sorted (pixel << 32 | poly) -> head flags of pixel groups
__global__ void k_multi_heads(const unsigned long long* __restrict__ m, int64_t M, int32_t* __restrict__ head) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < M; t += (int64_t)gridDim.x * kBT)
    head[t] = (t == 0 || (m[t] >> 32) != (m[t - 1] >> 32)) ? 1 : 0;
}

// head_scan = inclusive scan of heads: group index g = head_scan[t] - 1
__global__ void k_multi_records(const unsigned long long* __restrict__ m, int64_t M, const int32_t* __restrict__ hs,
                                int64_t NR, int32_t* __restrict__ sets, int2* __restrict__ set_rng,
                                RunRec* __restrict__ runs, int32_t* __restrict__ fine) {
  for (int64_t t = blockIdx.x * (int64_t)kBT + threadIdx.x; t < M; t += (int64_t)gridDim.x * kBT) {
    int32_t g = hs[t] - 1;
    sets[t] = (int32_t)(m[t] & 0xffffffffu);
    bool head = (t == 0 || (m[t] >> 32) != (m[t - 1] >> 32));
    if (!head) continue;
    int64_t e = t + 1;
    while (e < M && (m[e] >> 32) == (m[t] >> 32)) ++e;
    set_rng[g] = make_int2((int)t, (int)(e - t));
    runs[NR + g] = RunRec{0, 0, -2 - g};
    fine[(int64_t)(m[t] >> 32)] = -2 - (int32_t)(NR + g);
  }
}

__global__ void k_runs(int64_t NR, int W, const int64_t* __restrict__ run_end, const int32_t* __restrict__ run_cnt,
                       const int64_t* __restrict__ run_beg, const int32_t* __restrict__ fine, RunRec* __restrict__ runs) {
  for (int64_t r = blockIdx.x * (int64_t)kBT + threadIdx.x; r < NR; r += (int64_t)gridDim.x * kBT) {
    int64_t e = run_end[r];
    int32_t term = kEmpty;
    if ((int)(e % W) != W - 1) {
      int32_t v = fine[e + 1];                     // first non-boundary pixel right of the run
      if (v >= 0) term = v;
      else if (v <= -2) term = -2 - (int32_t)((-2 - (int64_t)v) - NR);   // multi record -> set index
    }
    runs[r] = RunRec{run_beg[r], run_cnt[r], term};
  }
}

__global__ void k_coarse(const int32_t* __restrict__ fine, int W, int H, int b, int Wc, int Hc,
                         uint16_t* __restrict__ coarse, unsigned long long* __restrict__ nmixed) {
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
    uint16_t c;
    if (uni && (int64_t)v0 + 1 < (int64_t)kTileMixed) c = (uint16_t)(v0 + 1);
    else { c = kTileMixed; atomicAdd(nmixed, 1ull); }
    coarse[t] = c;
  }
}

int bits_for(int64_t v) {  // bits to hold values 0..v
  int b = 1;
  while (b < 63 && (v >> b) != 0) ++b;
  return b;
}

struct DevBufs {
  std::vector<void*> ptrs;
  ~DevBufs() { for (void* p : ptrs) cudaFree(p); }
  template <class T> cudaError_t alloc(T** p, size_t count) {
    cudaError_t e = cudaMalloc((void**)p, std::max<size_t>(count, 1) * sizeof(T));
    if (e == cudaSuccess) ptrs.push_back(*p); else *p = nullptr;
    return e;
  }
  void release(void* p) {
    auto it = std::find(ptrs.begin(), ptrs.end(), p);
    if (it != ptrs.end()) { cudaFree(p); ptrs.erase(it); }
  }
};

int grid_for(int64_t n) {
  int64_t g = (n + kBT - 1) / kBT;
  int64_t cap = (int64_t)device_sm_count() * 8;
  return (int)imax64(1, std::min(g, cap));
}

#define SPADE_TRY(call, what)                                        \
  do {                                                               \
    cudaError_t _e = (call);                                         \
    if (_e != cudaSuccess) {                                         \
      return _e == cudaErrorMemoryAllocation                         \
                 ? set_error(SPADE_ERR_OOM, "%s: out of device memory", what) \
                 : check_cuda(_e, what);                             \
    }                                                                \
  } while (0)

#define LAUNCH(kern, n, st, ...)                                     \
  do {                                                               \
    kern<<<grid_for(n), kBT, 0, st>>>(__VA_ARGS__);                  \
    count_launch();                                                  \
    SPADE_TRY(cudaGetLastError(), #kern);                            \
  } while (0)

template <class F>
cudaError_t cub_call(DevBufs& bufs, cudaStream_t st, F f) {
  size_t tmp = 0;
  cudaError_t e = f(nullptr, tmp);
  if (e != cudaSuccess) return e;
  void* t = nullptr;
  e = bufs.alloc((char**)&t, tmp);
  if (e != cudaSuccess) return e;
  e = f(t, tmp);
  count_launch();
  (void)st;
  return e;
}

}  // namespace

int build_canvas(const int32_t* ring_xy, const int64_t* ring_off, const int64_t* poly_ring_off, int32_t P,
                 const spade_canvas_params* prm, cudaStream_t st, spade_canvas** out) {
  *out = nullptr;
  if (P < 0 || (P > 0 && (!ring_off || !poly_ring_off)))
    return set_error(SPADE_ERR_INVALID_ARG, "spade_build_canvas: bad polygon arguments");
  if (P > (1 << 30)) return set_error(SPADE_ERR_INVALID_ARG, "spade_build_canvas: too many polygons");
  int max_dim = 4096, forced_s = -1;
  if (prm) {
    if (prm->max_dim < 0 || prm->log2_pixel < -1 || prm->log2_pixel > 30)
      return set_error(SPADE_ERR_INVALID_ARG, "spade_build_canvas: bad canvas params");
    if (prm->max_dim > 0) max_dim = prm->max_dim;
    forced_s = prm->log2_pixel;
  }
  if (max_dim < 1 || max_dim > 65536) return set_error(SPADE_ERR_INVALID_ARG, "max_dim out of [1, 65536]");

  // --- offsets to the host for validation (R+1 and P+1 int64s) ---
  std::vector<int64_t> h_pro(P + 1, 0);
  if (P > 0) SPADE_TRY(cudaMemcpyAsync(h_pro.data(), poly_ring_off, sizeof(int64_t) * (P + 1), cudaMemcpyDeviceToHost, st), "copy poly_ring_off");
  SPADE_TRY(cudaStreamSynchronize(st), "sync");
  int64_t R = h_pro[P];
  if (h_pro[0] != 0 || R < 0) return set_error(SPADE_ERR_INVALID_ARG, "poly_ring_off must start at 0");
  for (int32_t p = 0; p < P; ++p)
    if (h_pro[p + 1] < h_pro[p]) return set_error(SPADE_ERR_INVALID_ARG, "poly_ring_off not non-decreasing at %d", p);
  std::vector<int64_t> h_ro(R + 1, 0);
  if (R > 0) {
    SPADE_TRY(cudaMemcpyAsync(h_ro.data(), ring_off, sizeof(int64_t) * (R + 1), cudaMemcpyDeviceToHost, st), "copy ring_off");
    SPADE_TRY(cudaStreamSynchronize(st), "sync");
  }
  int64_t V = h_ro[R];
  if (h_ro[0] != 0 || V < 0) return set_error(SPADE_ERR_INVALID_ARG, "ring_off must start at 0");
  for (int64_t r = 0; r < R; ++r)
    if (h_ro[r + 1] < h_ro[r]) return set_error(SPADE_ERR_INVALID_ARG, "ring_off not non-decreasing at %lld", (long long)r);
  if (V > 0 && !ring_xy) return set_error(SPADE_ERR_INVALID_ARG, "ring_xy is NULL");
  if (V >= (1ll << 31)) return set_error(SPADE_ERR_INVALID_ARG, "too many vertices");

  spade_canvas* c = new spade_canvas();
  cudaGetDevice(&c->device);
  c->d.num_polys = P;
  auto fail = [&](int code) { spade_canvas_free(c); return code; };
  if (V == 0) {  // no vertices: every point is outside every polygon
    c->empty = true;
    *out = c;
    return SPADE_OK;
  }

  DevBufs tmp;
  int4* seg; int32_t* epoly; int* ext; int* bad;
  if (tmp.alloc(&seg, V) || tmp.alloc(&epoly, V) || tmp.alloc(&ext, 4) || tmp.alloc(&bad, 1))
    return fail(set_error(SPADE_ERR_OOM, "build: edge buffers"));
  int h_ext0[4] = {INT_MAX, INT_MAX, INT_MIN, INT_MIN};
  int rc;
#define TRYF(call, what) do { cudaError_t _e = (call); if (_e != cudaSuccess) return fail(_e == cudaErrorMemoryAllocation ? set_error(SPADE_ERR_OOM, "%s", what) : check_cuda(_e, what)); } while (0)
  TRYF(cudaMemcpyAsync(ext, h_ext0, sizeof(h_ext0), cudaMemcpyHostToDevice, st), "ext init");
  TRYF(cudaMemsetAsync(bad, 0, sizeof(int), st), "memset");
  k_edges<<<grid_for(V), kBT, 0, st>>>((const int2*)ring_xy, ring_off, R, poly_ring_off, P, V, seg, epoly, ext, bad);
  count_launch();
  TRYF(cudaGetLastError(), "k_edges");
  int h_ext[4], h_bad = 0;
  TRYF(cudaMemcpyAsync(h_ext, ext, sizeof(h_ext), cudaMemcpyDeviceToHost, st), "ext");
  TRYF(cudaMemcpyAsync(&h_bad, bad, sizeof(int), cudaMemcpyDeviceToHost, st), "bad");
  TRYF(cudaStreamSynchronize(st), "sync edges");
  if (h_bad) return fail(set_error(SPADE_ERR_COORD_RANGE, "a polygon vertex lies outside [-2^30, 2^30)"));

  // --- canvas geometry (reading C5) ---
  int64_t ew = (int64_t)h_ext[2] - h_ext[0], eh = (int64_t)h_ext[3] - h_ext[1];
  int s = forced_s;
  if (s < 0) {
    s = 0;
    while (std::max((ew >> s) + 1, (eh >> s) + 1) > max_dim) ++s;
  }
  Geo g;
  g.minx = h_ext[0]; g.miny = h_ext[1]; g.s = s; g.S = 1ll << s;
  int64_t W64 = (ew >> s) + 1, H64 = (eh >> s) + 1;
  if (W64 * H64 > (1ll << 31) - 4) return fail(set_error(SPADE_ERR_INVALID_ARG, "canvas too large (%lld x %lld)", (long long)W64, (long long)H64));
  g.W = (int)W64; g.H = (int)H64;
  const int64_t WH = (int64_t)g.W * g.H;
  // coarse tiles: the shared-memory level holds at most kMaxTiles uint16 entries
  const int64_t kMaxTiles = 65536;
  int b = 0;
  while (((int64_t)(g.W + (1 << b) - 1) >> b) * ((int64_t)(g.H + (1 << b) - 1) >> b) > kMaxTiles) ++b;
  int Wc = (g.W + (1 << b) - 1) >> b, Hc = (g.H + (1 << b) - 1) >> b;

  // --- K-B1 counts, scans ---
  int64_t *nfrag, *nlist, *nev, *frag_off, *list_off, *ev_off;
  if (tmp.alloc(&nfrag, V) || tmp.alloc(&nlist, V) || tmp.alloc(&nev, V) || tmp.alloc(&frag_off, V + 1) ||
      tmp.alloc(&list_off, V + 1) || tmp.alloc(&ev_off, V + 1))
    return fail(set_error(SPADE_ERR_OOM, "build: count buffers"));
  k_count<<<grid_for(V), kBT, 0, st>>>(seg, V, g, nfrag, nlist, nev);
  count_launch();
  TRYF(cudaGetLastError(), "k_count");
  for (auto pr : {std::make_pair(nfrag, frag_off), std::make_pair(nlist, list_off), std::make_pair(nev, ev_off)}) {
    int64_t* in = pr.first; int64_t* o = pr.second;
    TRYF(cub_call(tmp, st, [&](void* t, size_t& sz) { return cub::DeviceScan::InclusiveSum(t, sz, in, o + 1, V, st); }), "scan counts");
    TRYF(cudaMemsetAsync(o, 0, sizeof(int64_t), st), "memset");
  }
  int64_t F = 0, L = 0, NE = 0;
  TRYF(cudaMemcpyAsync(&F, frag_off + V, 8, cudaMemcpyDeviceToHost, st), "F");
  TRYF(cudaMemcpyAsync(&L, list_off + V, 8, cudaMemcpyDeviceToHost, st), "L");
  TRYF(cudaMemcpyAsync(&NE, ev_off + V, 8, cudaMemcpyDeviceToHost, st), "NE");
  TRYF(cudaStreamSynchronize(st), "sync counts");
  tmp.release(nfrag); tmp.release(nlist); tmp.release(nev);

  const int pbits = bits_for(imax64(P - 1, 1)), cbits = bits_for(g.W - 1), jbits = bits_for(g.H - 1);
  if (pbits + cbits + jbits > 64) return fail(set_error(SPADE_ERR_INVALID_ARG, "canvas/polygon count too large for event keys"));

  Frag* frags; uint64_t* ev;
  if (tmp.alloc(&frags, F) || tmp.alloc(&ev, NE)) return fail(set_error(SPADE_ERR_OOM, "build: fragments"));
  k_emit<<<grid_for(V), kBT, 0, st>>>(seg, epoly, V, g, frag_off, ev_off, frags, ev, pbits, cbits);
  count_launch();
  TRYF(cudaGetLastError(), "k_emit");

  // --- mark boundary pixels, runs ---
  uint8_t* bmap; int32_t* scan;
  if (tmp.alloc(&bmap, WH) || tmp.alloc(&scan, WH)) return fail(set_error(SPADE_ERR_OOM, "build: bitmap"));
  if (cudaMalloc(&c->fine, sizeof(int32_t) * WH) != cudaSuccess) return fail(set_error(SPADE_ERR_OOM, "build: canvas"));
  TRYF(cudaMemsetAsync(bmap, 0, WH, st), "memset bmap");
  if (F > 0) { LAUNCH(k_mark, F, st, frags, F, g.W, bmap); }
  LAUNCH(k_run_flags, WH, st, bmap, WH, g.W, scan);
  TRYF(cub_call(tmp, st, [&](void* t, size_t& sz) { return cub::DeviceScan::InclusiveSum(t, sz, scan, scan, WH, st); }), "scan runs");
  int32_t NR32 = 0;
  TRYF(cudaMemcpyAsync(&NR32, scan + WH - 1, 4, cudaMemcpyDeviceToHost, st), "NR");
  TRYF(cudaStreamSynchronize(st), "sync runs");
  const int64_t NR = NR32;
  int64_t* run_end; int32_t* run_cnt; int64_t* run_beg;
  if (tmp.alloc(&run_end, NR) || tmp.alloc(&run_cnt, NR) || tmp.alloc(&run_beg, NR + 1))
    return fail(set_error(SPADE_ERR_OOM, "build: runs"));
  LAUNCH(k_run_ids, WH, st, bmap, scan, WH, g.W, c->fine, run_end);

  // --- run -> edge CSR, sorted by (run, polygon) ---
  uint64_t *lk, *lk2; int32_t *lv, *lv2;
  if (tmp.alloc(&lk, L) || tmp.alloc(&lk2, L) || tmp.alloc(&lv, L) || tmp.alloc(&lv2, L))
    return fail(set_error(SPADE_ERR_OOM, "build: run edges"));
  TRYF(cudaMemsetAsync(run_cnt, 0, sizeof(int32_t) * imax64(NR, 1), st), "memset");
  if (F > 0) { LAUNCH(k_list, F, st, frags, F, g.W, seg, epoly, scan, frag_off, list_off, lk, lv, run_cnt); }
  const int rbits = bits_for(imax64(NR - 1, 1));
  if (L > 0) {
    TRYF(cub_call(tmp, st, [&](void* t, size_t& sz) {
      return cub::DeviceRadixSort::SortPairs(t, sz, lk, lk2, lv, lv2, L, 0, 32 + rbits, st); }), "sort run edges");
  }
  if (NR > 0) {
    TRYF(cub_call(tmp, st, [&](void* t, size_t& sz) { return cub::DeviceScan::ExclusiveSum(t, sz, run_cnt, run_beg, NR, st); }), "scan run edges");
  }
  if (cudaMalloc(&c->run_seg, sizeof(int4) * imax64(L, 1)) != cudaSuccess ||
      cudaMalloc(&c->run_poly, sizeof(int32_t) * imax64(L, 1)) != cudaSuccess)
    return fail(set_error(SPADE_ERR_OOM, "build: run edge arrays"));
  if (L > 0) { LAUNCH(k_gather_edges, L, st, lv2, L, seg, epoly, c->run_seg, c->run_poly); }
  tmp.release(lk); tmp.release(lk2); tmp.release(lv); tmp.release(lv2);

  // --- K-B3 scanline fill ---
  uint64_t* ev2;
  if (tmp.alloc(&ev2, NE)) return fail(set_error(SPADE_ERR_OOM, "build: events"));
  if (NE > 0) {
    TRYF(cub_call(tmp, st, [&](void* t, size_t& sz) {
      return cub::DeviceRadixSort::SortKeys(t, sz, ev, ev2, NE, 0, jbits + pbits + cbits, st); }), "sort events");
  }
  tmp.release(ev);
  unsigned long long *multi = nullptr, *nmulti;
  int64_t multi_cap = 1 << 20;
  if (tmp.alloc(&nmulti, 1)) return fail(set_error(SPADE_ERR_OOM, "build: multi"));
  unsigned long long h_nmulti = 0;
  for (int attempt = 0; attempt < 2; ++attempt) {
    if (tmp.alloc(&multi, multi_cap)) return fail(set_error(SPADE_ERR_OOM, "build: multi list"));
    TRYF(cudaMemsetAsync(nmulti, 0, 8, st), "memset");
    TRYF(cudaMemsetAsync(bad, 0, 4, st), "memset");
    if (NE > 0) { LAUNCH(k_fill, (NE + 1) / 2, st, ev2, NE, g.W, pbits, cbits, bmap, c->fine, multi, nmulti, multi_cap, bad); }
    TRYF(cudaMemcpyAsync(&h_nmulti, nmulti, 8, cudaMemcpyDeviceToHost, st), "nmulti");
    TRYF(cudaMemcpyAsync(&h_bad, bad, 4, cudaMemcpyDeviceToHost, st), "bad");
    TRYF(cudaStreamSynchronize(st), "sync fill");
    if (h_bad) return fail(set_error(SPADE_ERR_INTERNAL, "scanline events do not pair up (flag %d)", h_bad));
    if ((int64_t)h_nmulti <= multi_cap) break;
    tmp.release(multi);
    multi_cap = (int64_t)h_nmulti;
    LAUNCH(k_reset_fill, WH, st, bmap, WH, c->fine);
  }
  const int64_t M = (int64_t)h_nmulti;
  int64_t NG = 0;
  if (M > 0) {
    unsigned long long* m2; int32_t* heads;
    if (tmp.alloc(&m2, M) || tmp.alloc(&heads, M)) return fail(set_error(SPADE_ERR_OOM, "build: multi sort"));
    TRYF(cub_call(tmp, st, [&](void* t, size_t& sz) { return cub::DeviceRadixSort::SortKeys(t, sz, multi, m2, M, 0, 64, st); }), "sort multi");
    LAUNCH(k_multi_heads, M, st, m2, M, heads);
    TRYF(cub_call(tmp, st, [&](void* t, size_t& sz) { return cub::DeviceScan::InclusiveSum(t, sz, heads, heads, M, st); }), "scan multi");
    int32_t ng32 = 0;
    TRYF(cudaMemcpyAsync(&ng32, heads + M - 1, 4, cudaMemcpyDeviceToHost, st), "NG");
    TRYF(cudaStreamSynchronize(st), "sync multi");
    NG = ng32;
    if (cudaMalloc(&c->sets, sizeof(int32_t) * M) != cudaSuccess || cudaMalloc(&c->set_rng, sizeof(int2) * NG) != cudaSuccess ||
        cudaMalloc(&c->runs, sizeof(RunRec) * (NR + NG)) != cudaSuccess)
      return fail(set_error(SPADE_ERR_OOM, "build: records"));
    LAUNCH(k_multi_records, M, st, m2, M, heads, NR, c->sets, c->set_rng, c->runs, c->fine);
  } else {
    if (cudaMalloc(&c->runs, sizeof(RunRec) * imax64(NR, 1)) != cudaSuccess)
      return fail(set_error(SPADE_ERR_OOM, "build: records"));
  }
  if (NR > 0) { LAUNCH(k_runs, NR, st, NR, g.W, run_end, run_cnt, run_beg, c->fine, c->runs); }

  // --- K-B5 coarse tiles ---
  if (cudaMalloc(&c->coarse, sizeof(uint16_t) * ((int64_t)Wc * Hc + 16)) != cudaSuccess)
    return fail(set_error(SPADE_ERR_OOM, "build: coarse"));
  TRYF(cudaMemsetAsync(nmulti, 0, 8, st), "memset");
  LAUNCH(k_coarse, (int64_t)Wc * Hc, st, c->fine, g.W, g.H, b, Wc, Hc, c->coarse, nmulti);
  unsigned long long h_mixed = 0;
  TRYF(cudaMemcpyAsync(&h_mixed, nmulti, 8, cudaMemcpyDeviceToHost, st), "mixed");
  TRYF(cudaStreamSynchronize(st), "sync coarse");
#undef TRYF

  c->empty = false;
  c->num_runs = NR;
  c->num_records = NR + NG;
  c->num_run_edges = L;
  c->num_set_entries = M;
  c->mixed_tile_frac = (double)h_mixed / ((double)Wc * Hc);
  CanvasDev& d = c->d;
  d.minx = (int32_t)g.minx; d.miny = (int32_t)g.miny;
  d.extw = (uint32_t)ew; d.exth = (uint32_t)eh;
  d.s = s; d.W = g.W; d.H = g.H; d.b = b; d.Wc = Wc; d.Hc = Hc;
  d.fine = c->fine; d.coarse = c->coarse; d.runs = c->runs; d.run_seg = c->run_seg; d.run_poly = c->run_poly;
  d.sets = c->sets; d.set_rng = c->set_rng;
  (void)rc;
  *out = c;
  return SPADE_OK;
}

}  // namespace spade
