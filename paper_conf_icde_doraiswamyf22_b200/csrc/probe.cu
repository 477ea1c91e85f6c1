// probe.cu — the point probe (the metric kernel): stream points, look them up in the canvas, run
// the exact test only for points on boundary pixels, and aggregate / emit results.
//
// Paper: single rendering pass over the points with blend + mask + map fused in one fragment
// shader (Sec. 5.1-5.2); the constraint canvas kept in fast read-only memory
// (P:163); points on boundary pixels get the exact test through the boundary index (P:146,
// Fig. 4); COUNT by additive blending of partial aggregates, plan 2 for points;
// Map output via a unique slot per result + scan.
//
// B200 design:
//   * one persistent CTA per SM, T threads; the coarse canvas (<= 80K uint16 tiles) is copied
//     into shared memory once per CTA, so most points are classified by ONE LDS;
//   * points stream with 256-bit loads (LDG.E.256, L1::no_allocate, L2::evict_first);
//   * points in mixed tiles gather one int32 fine pixel from L2 (evict_last policy); all gathers of
//     a thread's batch are issued before any is consumed (memory-level parallelism);
//   * boundary points are compacted per warp (ballot) into a shared-memory queue and evaluated
//     32 at a time (one per lane) against the few edges touching their pixel (exact int64 tests);
//   * COUNT: shared-memory per-polygon histogram (smem atomics), flushed once per CTA with
//     64-bit global atomics; SELECT/PAIRS: CTA-aggregated output reservation (one global atomic
//     per CTA batch) and direct stores.
#include <cstdint>
#include <algorithm>
#include "spade_internal.cuh"

namespace spade {

namespace {

enum Mode { kCountSmem = 0, kCountGlobal = 1, kSelect = 2, kPairs = 3 };
constexpr int kQCap = 64;          // per-warp boundary queue entries (drained at >= 32)

struct alignas(32) Vec4 { int4 a, b; };   // 4 points
struct alignas(16) QEntry { int x, y, rec; uint32_t pidx; };

__device__ __forceinline__ Vec4 ld_stream(const Vec4* p) {
  Vec4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r.a.x), "=r"(r.a.y), "=r"(r.a.z), "=r"(r.a.w), "=r"(r.b.x), "=r"(r.b.y), "=r"(r.b.z),
                 "=r"(r.b.w)
               : "l"(p));
  return r;
}

__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ uint32_t ld_fine(const int32_t* p, uint64_t pol) {
  uint32_t r;
  asm volatile("ld.global.nc.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
  return r;
}

// Output side of a launch (what the sinks write).
struct Out {
  unsigned long long* counts; // COUNT
  unsigned long long* total;  // SELECT/PAIRS: number of results (may exceed capacity)
  int64_t* out_ids;           // SELECT ids / PAIRS point ids
  int32_t* out_poly;          // PAIRS polygon ids
  int64_t cap;
  int64_t id_base;            // point id of xy[0]
};

struct Params {
  CanvasDev cv;
  const CanvasDev* cvg;       // the same, in global memory (for the out-of-line exact test)
  const int2* xy;
  int64_t n;
  int64_t head;               // points before the first 32-byte aligned one (0..3)
  int64_t nvec;               // aligned 4-point vectors after the head
  Out o;
};

// classification of one point before the fine gather:
//   0 = no polygon, 1..2^31-1 = owner + 1, bit31 set = needs the fine pixel (index in low 31 bits)
__device__ __forceinline__ uint32_t classify_coarse(const CanvasDev& cv, const uint16_t* tiles, int x, int y) {
  uint32_t ux = (uint32_t)x - (uint32_t)cv.minx, uy = (uint32_t)y - (uint32_t)cv.miny;
  if (ux > cv.extw || uy > cv.exth) return 0u;
  uint32_t fx = ux >> cv.s, fy = uy >> cv.s;
  uint32_t t = tiles[(fy >> cv.b) * (uint32_t)cv.Wc + (fx >> cv.b)];
  if (t != kTileMixed) return t;
  return 0x80000000u | (fy * (uint32_t)cv.W + fx);
}
// after the gather: 0 = none, owner+1, or bit31 | record id (boundary pixel / multi-owner pixel)
__device__ __forceinline__ uint32_t classify_fine(int32_t v) {
  return v >= 0 ? (uint32_t)v + 1u : (v == kEmpty ? 0u : (0x80000000u | (uint32_t)(-2 - v)));
}

// Pixel-local exact test of one edge for point p in the pixel whose left side is x = X
// (DESIGN.md "Canvas"):  cu(X, py) ^ cr(X, py) ^ cr(px, py), where cr is the half-open rightward
// ray test of reading C1 and cu the upward ray test of the same perturbation.  Both share the
// cross product o at (X, py).  Exact in int64 (all coordinates in [-2^30, 2^30)).
__device__ __forceinline__ int local_bit(int4 e, int X, int px, int py) {
  const int dx = e.z - e.x, dy = e.w - e.y;
  const long long o = (long long)dx * (py - e.y) - (long long)dy * (X - e.x);
  const long long o2 = o - (long long)dy * (px - X);
  const bool ys = (e.y > py) != (e.w > py);
  const bool xs = (e.x > X) != (e.z > X);
  const bool crX = ys && (dy > 0 ? o > 0 : o < 0);
  const bool crP = ys && (dy > 0 ? o2 > 0 : o2 < 0);
  const bool cuX = xs && (dx > 0 ? (o < 0 || (o == 0 && dy > 0)) : (o > 0 || (o == 0 && dy < 0)));
  return (int)(crX ^ crP ^ cuX);
}

// Exact point-in-polygon for a point on boundary pixel (or multi-owner pixel) record `rec`:
//   inside(p, P) = [P in K] XOR parity_P(local_bit over P's edges touching the pixel)
// emit(P) is called for every polygon containing the point, in increasing polygon order.
template <class Emit>
__device__ __forceinline__ void pip_eval(const CanvasDev* __restrict__ cv, int px, int py, uint32_t rec, Emit&& emit) {
  const RunRec r = cv->runs[rec];
  const int X = cv->minx + (int)((((uint32_t)px - (uint32_t)cv->minx) >> cv->s) << cv->s);
  int tn, tb = 0;
  const bool tsingle = r.term >= 0;
  if (tsingle) tn = 1;
  else if (r.term == kEmpty) tn = 0;
  else { int2 g = cv->set_rng[-2 - r.term]; tb = g.x; tn = g.y; }
  const int32_t* sets = cv->sets;
  auto term_at = [&](int i) { return tsingle ? r.term : sets[tb + i]; };
  int ti = 0;
  auto finalize = [&](int P, int par) {
    while (ti < tn && term_at(ti) < P) emit(term_at(ti++));
    if (ti < tn && term_at(ti) == P) { par ^= 1; ++ti; }
    if (par) emit(P);
  };
  const int4* seg = cv->run_seg;
  const int32_t* poly = cv->run_poly;
  int cur = -1, par = 0;
  const int64_t e1 = r.edge_begin + r.edge_cnt;
  for (int64_t e = r.edge_begin; e < e1; ++e) {
    const int p = __ldg(poly + e);
    if (p != cur) {
      if (cur >= 0) finalize(cur, par);
      cur = p; par = 0;
    }
    par ^= local_bit(__ldg(seg + e), X, px, py);
  }
  if (cur >= 0) finalize(cur, par);
  while (ti < tn) emit(term_at(ti++));
}

template <int MODE>
__device__ __forceinline__ void count_hit(unsigned int* hist, unsigned long long* counts, int owner) {
  if (MODE == kCountSmem) atomicAdd(&hist[owner], 1u);
  else atomicAdd(counts + owner, 1ull);
}

// Emission from the rare paths (boundary queue drains, unaligned head/tail): per-lane atomics.
template <int MODE>
__device__ __forceinline__ void rare_emit_point(const CanvasDev* __restrict__ cvg, unsigned int* hist, const Out& o,
                                                int x, int y, uint32_t rec, int64_t pid) {
  if (MODE == kCountSmem || MODE == kCountGlobal) {
    pip_eval(cvg, x, y, rec, [&](int p) { count_hit<MODE>(hist, o.counts, p); });
  } else if (MODE == kSelect) {
    bool any = false;
    pip_eval(cvg, x, y, rec, [&](int) { any = true; });
    if (any) {
      unsigned long long q = atomicAdd(o.total, 1ull);
      if ((int64_t)q < o.cap) o.out_ids[q] = pid;
    }
  } else {
    pip_eval(cvg, x, y, rec, [&](int p) {
      unsigned long long q = atomicAdd(o.total, 1ull);
      if ((int64_t)q < o.cap) { o.out_ids[q] = pid; o.out_poly[q] = p; }
    });
  }
}

template <int MODE>
__device__ __forceinline__ void rare_emit_owner(unsigned int* hist, const Out& o, int owner, int64_t pid) {
  if (MODE == kCountSmem || MODE == kCountGlobal) count_hit<MODE>(hist, o.counts, owner);
  else {
    unsigned long long q = atomicAdd(o.total, 1ull);
    if ((int64_t)q < o.cap) {
      o.out_ids[q] = pid;
      if (MODE == kPairs) o.out_poly[q] = owner;
    }
  }
}

// One scalar point (unaligned head / tail): classify synchronously.
template <int MODE>
__device__ __noinline__ void scalar_point(const CanvasDev* __restrict__ cvg, const uint16_t* tiles, unsigned int* hist,
                                          Out o, int x, int y, int64_t pid) {
  const CanvasDev cv = *cvg;
  uint32_t c = classify_coarse(cv, tiles, x, y);
  if (c & 0x80000000u) c = classify_fine(cv.fine[c & 0x7fffffffu]);
  if (c == 0) return;
  if (c & 0x80000000u) rare_emit_point<MODE>(cvg, hist, o, x, y, c & 0x7fffffffu, pid);
  else rare_emit_owner<MODE>(hist, o, (int)c - 1, pid);
}

// Evaluate up to 32 queued boundary points (one per lane).  Out of line: it is the rare path and
// keeping it out of the streaming loop keeps that loop's register footprint small.
template <int MODE>
__device__ __noinline__ void drain(const CanvasDev* __restrict__ cvg, const QEntry* wq, int cnt, int lane,
                                   unsigned int* hist, Out o) {
  if (lane < cnt) {
    const QEntry e = wq[lane];
    rare_emit_point<MODE>(cvg, hist, o, e.x, e.y, (uint32_t)e.rec, o.id_base + (int64_t)e.pidx);
  }
}

template <int MODE, int T, int U>
__global__ void __launch_bounds__(T, 1) k_probe(const __grid_constant__ Params prm) {
  extern __shared__ __align__(16) unsigned char smem[];
  const CanvasDev& cv = prm.cv;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int NW = T / 32;
  const int ntiles = cv.Wc * cv.Hc;
  const int tiles_bytes = ((ntiles * 2) + 15) & ~15;
  uint16_t* tiles = (uint16_t*)smem;
  QEntry* queues = (QEntry*)(smem + tiles_bytes);
  unsigned char* rest = smem + tiles_bytes + NW * kQCap * sizeof(QEntry);
  unsigned int* hist = (unsigned int*)rest;               // COUNT (smem histogram)
  int* s_scan = (int*)rest;                               // SELECT/PAIRS: [NW] warp sums
  long long* s_base = (long long*)(rest + 128 * sizeof(int));   // [NW] warp output bases

  for (int i = tid; i < tiles_bytes / 16; i += T) ((int4*)tiles)[i] = __ldg((const int4*)cv.coarse + i);
  if (MODE == kCountSmem)
    for (int i = tid; i < cv.num_polys; i += T) hist[i] = 0u;
  __syncthreads();

  QEntry* wq = queues + warp * kQCap;
  int qn = 0;                                   // warp-uniform
  const uint64_t pol = policy_evict_last();

  // unaligned head and tail (< 8 points): CTA 0, warp 0
  if (blockIdx.x == 0 && warp == 0) {
    const int64_t tail0 = prm.head + 4 * prm.nvec;
    const int64_t ntail = prm.n - tail0;
    if (lane < prm.head) {
      const int2 p = prm.xy[lane];
      scalar_point<MODE>(prm.cvg, tiles, hist, prm.o, p.x, p.y, prm.o.id_base + lane);
    } else if (lane >= 4 && lane - 4 < ntail) {
      const int64_t i = tail0 + (lane - 4);
      const int2 p = prm.xy[i];
      scalar_point<MODE>(prm.cvg, tiles, hist, prm.o, p.x, p.y, prm.o.id_base + i);
    }
  }

  const Vec4* vp = (const Vec4*)(prm.xy + prm.head);
  const int64_t chunk = (int64_t)T * U;
  for (int64_t base = (int64_t)blockIdx.x * chunk; base < prm.nvec; base += (int64_t)gridDim.x * chunk) {
    Vec4 v[U];
#pragma unroll
    for (int k = 0; k < U; ++k) {
      const int64_t idx = base + (int64_t)k * T + tid;
      if (idx < prm.nvec) v[k] = ld_stream(vp + idx);
      else { v[k].a = make_int4(INT32_MIN, INT32_MIN, INT32_MIN, INT32_MIN); v[k].b = v[k].a; }
    }
    // phase A: coarse (shared memory) classification.  Padding points (INT32_MIN) are outside
    // every valid extent (vertices are >= -2^30), so they classify as 0.
    uint32_t c[4 * U];
    uint32_t mix = 0;
#pragma unroll
    for (int k = 0; k < U; ++k) {
      c[4 * k + 0] = classify_coarse(cv, tiles, v[k].a.x, v[k].a.y);
      c[4 * k + 1] = classify_coarse(cv, tiles, v[k].a.z, v[k].a.w);
      c[4 * k + 2] = classify_coarse(cv, tiles, v[k].b.x, v[k].b.y);
      c[4 * k + 3] = classify_coarse(cv, tiles, v[k].b.z, v[k].b.w);
    }
#pragma unroll
    for (int q = 0; q < 4 * U; ++q) mix |= (c[q] >> 31) << q;
    // phase B: all fine-pixel gathers of the batch in flight together
    if (mix) {
#pragma unroll
      for (int q = 0; q < 4 * U; ++q)
        if ((mix >> q) & 1u) c[q] = ld_fine(cv.fine + (c[q] & 0x7fffffffu), pol);
#pragma unroll
      for (int q = 0; q < 4 * U; ++q)
        if ((mix >> q) & 1u) c[q] = classify_fine((int32_t)c[q]);
    }
    // phase C1: boundary points -> warp queue (ballot compaction), drained 32 at a time
    uint32_t bnd = 0;
#pragma unroll
    for (int q = 0; q < 4 * U; ++q) bnd |= (c[q] >> 31) << q;
    if (__any_sync(0xffffffffu, bnd != 0u)) {
#pragma unroll
      for (int q = 0; q < 4 * U; ++q) {
        const bool isb = (bnd >> q) & 1u;
        const unsigned m = __ballot_sync(0xffffffffu, isb);
        if (m) {
          if (isb) {
            const int k = q >> 2, h = q & 3;
            const int x = h == 0 ? v[k].a.x : h == 1 ? v[k].a.z : h == 2 ? v[k].b.x : v[k].b.z;
            const int y = h == 0 ? v[k].a.y : h == 1 ? v[k].a.w : h == 2 ? v[k].b.y : v[k].b.w;
            const int64_t pidx = prm.head + 4 * (base + (int64_t)k * T + tid) + h;
            wq[qn + __popc(m & ((1u << lane) - 1u))] = QEntry{x, y, (int)(c[q] & 0x7fffffffu), (uint32_t)pidx};
          }
          qn += __popc(m);
          if (qn >= 32) {
            __syncwarp();
            drain<MODE>(prm.cvg, wq, 32, lane, hist, prm.o);
            __syncwarp();
            if (lane < qn - 32) wq[lane] = wq[32 + lane];
            __syncwarp();
            qn -= 32;
          }
        }
      }
    }
    // phase C2: direct hits
    if (MODE == kCountSmem || MODE == kCountGlobal) {
#pragma unroll
      for (int q = 0; q < 4 * U; ++q)
        if (c[q] != 0u && !(c[q] >> 31)) count_hit<MODE>(hist, prm.o.counts, (int)c[q] - 1);
    } else {
      // CTA-aggregated reservation of output slots for this batch (Map with a scan)
      int h = 0;
#pragma unroll
      for (int q = 0; q < 4 * U; ++q) h += (c[q] != 0u && !(c[q] >> 31)) ? 1 : 0;
      int incl = h;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        int t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
      }
      if (lane == 31) s_scan[warp] = incl;
      __syncthreads();
      if (warp == 0) {
        int wsum = lane < NW ? s_scan[lane] : 0, wincl = wsum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          int t = __shfl_up_sync(0xffffffffu, wincl, o);
          if (lane >= o) wincl += t;
        }
        unsigned long long gb = 0;
        if (lane == 31 && wincl > 0) gb = atomicAdd(prm.o.total, (unsigned long long)wincl);
        gb = __shfl_sync(0xffffffffu, gb, 31);
        if (lane < NW) s_base[lane] = (long long)gb + (wincl - wsum);
      }
      __syncthreads();
      int64_t pos = s_base[warp] + (incl - h);
#pragma unroll
      for (int q = 0; q < 4 * U; ++q) {
        if (c[q] != 0u && !(c[q] >> 31)) {
          if (pos < prm.o.cap) {
            const int k = q >> 2, hh = q & 3;
            prm.o.out_ids[pos] = prm.o.id_base + prm.head + 4 * (base + (int64_t)k * T + tid) + hh;
            if (MODE == kPairs) prm.o.out_poly[pos] = (int)c[q] - 1;
          }
          ++pos;
        }
      }
      __syncthreads();   // s_scan / s_base reuse next batch
    }
  }
  if (qn > 0) {
    __syncwarp();
    drain<MODE>(prm.cvg, wq, qn, lane, hist, prm.o);
  }
  if (MODE == kCountSmem) {
    __syncthreads();
    for (int i = tid; i < cv.num_polys; i += T)
      if (hist[i]) atomicAdd(prm.o.counts + i, (unsigned long long)hist[i]);
  }
}

template <int MODE, int T, int U>
int launch(const spade_canvas* c, const int2* xy, int64_t n, const Params& base, size_t extra_smem, cudaStream_t st) {
  const int ntiles = c->d.Wc * c->d.Hc;
  const size_t smem = (((size_t)ntiles * 2 + 15) & ~(size_t)15) + (T / 32) * kQCap * sizeof(QEntry) + extra_smem;
  auto kern = k_probe<MODE, T, U>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return check_cuda(e, "probe smem attribute");
  const int sms = device_sm_count();
  // launches of at most 2^31 points (queue entries hold 32-bit point offsets)
  const int64_t kMax = 1ll << 31;
  for (int64_t off = 0; off < n; off += kMax) {
    const int64_t m = std::min(kMax, n - off);
    Params p = base;
    p.xy = xy + off;
    p.n = m;
    const uintptr_t addr = (uintptr_t)p.xy;
    p.head = std::min<int64_t>(m, (int64_t)(((32 - (addr & 31)) & 31) / 8));
    p.nvec = (m - p.head) / 4;
    p.o.id_base = base.o.id_base + off;
    const int64_t chunks = (p.nvec + (int64_t)T * U - 1) / ((int64_t)T * U);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(sms, chunks));
    kern<<<grid, T, smem, st>>>(p);
    count_launch();
    e = cudaGetLastError();
    if (e != cudaSuccess) return check_cuda(e, "probe launch");
  }
  return SPADE_OK;
}

constexpr size_t kSmemBudget = 227 * 1024;
constexpr int kT = 1024, kU = 2;          // COUNT / SELECT (<= 64 registers per thread)
constexpr int kTP = 1024, kUP = 2;        // PAIRS

Params base_params(const spade_canvas* c) {
  Params p{};
  p.cv = c->d;
  p.cvg = c->d_dev;
  return p;
}

}  // namespace

int launch_count(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t* counts, cudaStream_t st) {
  if (c->empty || n == 0) return SPADE_OK;
  Params p = base_params(c);
  p.o.counts = (unsigned long long*)counts;
  const size_t fixed = (((size_t)c->d.Wc * c->d.Hc * 2 + 15) & ~(size_t)15) + (kT / 32) * kQCap * sizeof(QEntry);
  const size_t hist = (size_t)c->d.num_polys * 4;
  if (fixed + hist <= kSmemBudget) return launch<kCountSmem, kT, kU>(c, (const int2*)xy, n, p, hist, st);
  return launch<kCountGlobal, kT, kU>(c, (const int2*)xy, n, p, 0, st);
}

int launch_select(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t base, int64_t* out, int64_t cap,
                  unsigned long long* d_total, cudaStream_t st) {
  if (c->empty || n == 0) return SPADE_OK;
  Params p = base_params(c);
  p.o.id_base = base; p.o.out_ids = out; p.o.cap = cap; p.o.total = d_total;
  return launch<kSelect, kT, kU>(c, (const int2*)xy, n, p, 128 * sizeof(int) + 32 * sizeof(long long), st);
}

int launch_pairs(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t base, int64_t* opt, int32_t* opl,
                 int64_t cap, unsigned long long* d_total, cudaStream_t st) {
  if (c->empty || n == 0) return SPADE_OK;
  Params p = base_params(c);
  p.o.id_base = base; p.o.out_ids = opt; p.o.out_poly = opl; p.o.cap = cap; p.o.total = d_total;
  return launch<kPairs, kTP, kUP>(c, (const int2*)xy, n, p, 128 * sizeof(int) + 32 * sizeof(long long), st);
}

}  // namespace spade
