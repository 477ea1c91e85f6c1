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
#include <cstdlib>
#include <cub/block/block_scan.cuh>
#include "spade_internal.cuh"

namespace spade {

namespace {

enum Mode { kCountSmem = 0, kCountGlobal = 1, kSelect = 2, kPairs = 3 };

struct alignas(32) Vec4 { int4 a, b; };   // 4 points
struct alignas(8) QEntry { uint32_t rec, pidx; };   // boundary point: record and point index

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

// Deferred boundary point (the exact test runs in a second, load-balanced kernel).
struct alignas(16) DEntry { int x, y; uint32_t rec, pidx; };
constexpr uint32_t kHole = 0xffffffffu;   // DEntry.rec of a reserved-but-unused slot

struct Params {
  CanvasDev cv;
  DEntry* defer;              // per-CTA regions of defer_cap entries (nullptr: drain in-loop)
  uint32_t defer_cap;
  unsigned int* defer_fill;   // [grid] entries used per CTA region
  const CanvasDev* cvg;       // the same, in global memory (for the out-of-line exact test)
  const int2* xy;
  int64_t n;
  int64_t head;               // points before the first 32-byte aligned one (0..3)
  int64_t nvec;               // aligned 4-point vectors after the head
  Out o;
};

// Point class c after the fine gather: c = fine pixel value + 1, i.e. 0 = no polygon,
// 1 .. 2^31-1 = owner + 1, and >= 2^31 = record ~c (boundary / multi-owner pixel).  Uniform
// coarse tiles give the same encoding directly (tile value = owner + 1, 0 = empty).
__device__ __forceinline__ uint32_t classify_fine(int32_t v) { return (uint32_t)v + 1u; }

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
  const uint32_t ux = (uint32_t)x - (uint32_t)cv.minx, uy = (uint32_t)y - (uint32_t)cv.miny;
  if (ux > cv.extw || uy > cv.exth) return;
  const uint32_t fx = ux >> cv.s, fy = uy >> cv.s;
  uint32_t c = tiles[(fy >> cv.b) * (uint32_t)(cv.Wc + 1) + (fx >> cv.b)];
  if (c >= cv.mix_min) c = classify_fine(*fine_ptr(cv, c, fx, fy));
  if (c == 0) return;
  if (c & 0x80000000u) rare_emit_point<MODE>(cvg, hist, o, x, y, ~c, pid);
  else rare_emit_owner<MODE>(hist, o, (int)c - 1, pid);
}

// Evaluate up to 32 queued boundary points (one per lane).  Out of line: it is the rare path and
// keeping it out of the streaming loop keeps that loop's register footprint small.  Queue entries
// are 8 B (record, point index): a small queue leaves more of the SM's 256 KB for L1, which caches
// the fine-pixel gathers of clustered points.
template <int MODE>
__device__ __noinline__ void drain(const CanvasDev* __restrict__ cvg, const int2* __restrict__ xy, const QEntry* wq,
                                   int cnt, int lane, unsigned int* hist, Out o) {
  const bool active = lane < cnt;
  QEntry e{0u, 0u};
  int2 p = make_int2(0, 0);
  if (active) {
    e = wq[lane];
    p = __ldg(xy + e.pidx);                     // re-read here (rare) so the streaming loop never waits
  }
  const int64_t pid = o.id_base + (int64_t)e.pidx;
  if (MODE == kCountSmem || MODE == kCountGlobal) {
    if (active) pip_eval(cvg, p.x, p.y, e.rec, [&](int q) { count_hit<MODE>(hist, o.counts, q); });
    return;
  }
  // SELECT / PAIRS: count this lane's results, reserve all of the warp's slots with ONE global
  // atomic (a per-result atomic on the single counter serialises badly), then write them.
  int nres = 0;
  if (active) {
    if (MODE == kSelect) { bool any = false; pip_eval(cvg, p.x, p.y, e.rec, [&](int) { any = true; }); nres = any; }
    else pip_eval(cvg, p.x, p.y, e.rec, [&](int) { ++nres; });
  }
  int incl = nres;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int t = __shfl_up_sync(0xffffffffu, incl, d);
    if (lane >= d) incl += t;
  }
  unsigned long long gb = 0;
  if (lane == 31 && incl > 0) gb = atomicAdd(o.total, (unsigned long long)incl);
  gb = __shfl_sync(0xffffffffu, gb, 31);
  int64_t pos = (int64_t)gb + (incl - nres);
  if (nres) {
    if (MODE == kSelect) {
      if (pos < o.cap) o.out_ids[pos] = pid;
    } else {
      pip_eval(cvg, p.x, p.y, e.rec, [&](int q) {
        if (pos < o.cap) { o.out_ids[pos] = pid; o.out_poly[pos] = q; }
        ++pos;
      });
    }
  }
}

// Per-CTA shared-memory layout (bytes, in order):
//   tiles   (Wc+1) x (Hc+1) uint16 (pitch Wc+1), rounded up to 16 B; the last column and row are
//           always-empty sentinels: tile coordinates are clamped into them (no extent test)
//   queues  NW * (32 + 128 U) QEntry (8 B; boundary points per warp).  Keep the total <= ~196 KB:
//           measured, the probe loses ~35% when the L1 carve-out left over drops below ~60 KB.
//   COUNT   kHC copies of (P + 1) uint32 bins (bin P = "no polygon" trash bin)
//   SELECT/PAIRS: 128 int warp sums + 32 int64 warp bases
constexpr int kHC = 8;             // histogram copies (lane & 7): spreads same-polygon atomics

__host__ __device__ constexpr int qcap_for(int U) { return 32 + 32 * 4 * U; }
// tile array incl. the sentinel column and row, rounded up to 16 B
__host__ __device__ __forceinline__ size_t tiles_bytes_for(int Wc, int Hc) { return (((size_t)(Wc + 1) * (Hc + 1)) * 2 + 15) & ~(size_t)15; }

template <int MODE, int T, int U, int PF, int COMPACT>
__global__ void __launch_bounds__(T, 1) k_probe(const __grid_constant__ Params prm) {
  extern __shared__ __align__(16) unsigned char smem[];
  const CanvasDev& cv = prm.cv;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int NW = T / 32;
  constexpr int NPT = 4 * U;                      // points per thread per batch

  const uint32_t tbytes = (uint32_t)tiles_bytes_for(cv.Wc, cv.Hc);
  uint16_t* tiles = (uint16_t*)smem;
  QEntry* queues = (QEntry*)(smem + tbytes);
  unsigned char* rest = smem + tbytes + NW * qcap_for(U) * sizeof(QEntry);
  const uint32_t P = (uint32_t)cv.num_polys;
  unsigned int* hist = (unsigned int*)rest;                       // COUNT
  unsigned int* myhist = hist + (lane & (kHC - 1)) * (P + 1);
  int* s_scan = (int*)rest;                                       // SELECT/PAIRS
  long long* s_base = (long long*)(rest + 128 * sizeof(int));

  for (uint32_t i = tid; i < tbytes / 16; i += T) ((int4*)tiles)[i] = __ldg((const int4*)cv.coarse + i);
  if (MODE == kCountSmem)
    for (uint32_t i = tid; i < kHC * (P + 1); i += T) hist[i] = 0u;
  __syncthreads();

  QEntry* wq = queues + warp * qcap_for(U);
  __shared__ int s_qn[NW];                      // per-warp queue fill
  __shared__ unsigned int s_dfill;              // deferred entries reserved by this CTA
  if (lane == 0) s_qn[warp] = 0;
  if (tid == 0) s_dfill = 0;
  __syncthreads();
  DEntry* const dreg = prm.defer ? prm.defer + (size_t)blockIdx.x * prm.defer_cap : nullptr;
  const uint64_t pol = policy_evict_last();

  // unaligned head and tail (< 8 points): CTA 0, warp 0
  if (blockIdx.x == 0 && warp == 0) {
    const int64_t tail0 = prm.head + 4 * prm.nvec;
    const int64_t ntail = prm.n - tail0;
    if (lane < prm.head) {
      const int2 p = prm.xy[lane];
      scalar_point<MODE>(prm.cvg, tiles, myhist, prm.o, p.x, p.y, prm.o.id_base + lane);
    } else if (lane >= 4 && lane - 4 < ntail) {
      const int64_t i = tail0 + (lane - 4);
      const int2 p = prm.xy[i];
      scalar_point<MODE>(prm.cvg, tiles, myhist, prm.o, p.x, p.y, prm.o.id_base + i);
    }
  }

  const Vec4* vp = (const Vec4*)(prm.xy + prm.head);
  const uint32_t nvec = (uint32_t)prm.nvec;      // launches hold < 2^31 points
  const uint32_t chunk = (uint32_t)(T * U);
  const uint32_t minx = (uint32_t)cv.minx, miny = (uint32_t)cv.miny;
  const uint32_t sb = (uint32_t)(cv.s + cv.b), s = (uint32_t)cv.s, Wc = (uint32_t)cv.Wc, W = (uint32_t)cv.W;
  const uint32_t Hc = (uint32_t)cv.Hc, Wc1 = Wc + 1u;
  const uint32_t b = (uint32_t)cv.b, bm = (1u << cv.b) - 1u, mixmin = cv.mix_min;
  const int32_t* __restrict__ finep = COMPACT ? cv.cfine : cv.fine;
  auto load_batch = [&](Vec4 (&v)[U], uint32_t base) {
    if (base + chunk <= nvec) {                  // CTA-uniform: full batch, no bounds checks
#pragma unroll
      for (int k = 0; k < U; ++k) v[k] = ld_stream(vp + base + k * T + tid);
    } else {
#pragma unroll
      for (int k = 0; k < U; ++k) {
        const uint32_t idx = base + k * T + tid;
        if (idx < nvec) v[k] = ld_stream(vp + idx);
        else { v[k].a = make_int4(INT32_MIN, INT32_MIN, INT32_MIN, INT32_MIN); v[k].b = v[k].a; }
      }
    }
  };
  const uint32_t stride = gridDim.x * chunk;
  Vec4 nxt[U];
  if (PF && blockIdx.x * chunk < nvec) load_batch(nxt, blockIdx.x * chunk);
  for (uint32_t base = blockIdx.x * chunk; base < nvec; base += stride) {
    Vec4 v[U];
    if (PF) {
#pragma unroll
      for (int k = 0; k < U; ++k) v[k] = nxt[k];
      if (base + stride < nvec) load_batch(nxt, base + stride);   // next batch in flight while this one is processed
    } else {
      load_batch(v, base);
    }
    // phase A: coarse (shared memory) lookup, branch-free.  Offsets from the extent origin are
    // unsigned; points left of / below the origin wrap to huge values and, like points right of /
    // above the canvas, clamp into the always-empty sentinel column / row (exact because
    // 2^(s+b) <= 2^30, see canvas_build.cu).  c = 0 (none) | owner + 1 | tile value (mixed).
    uint32_t c[NPT];
#pragma unroll
    for (int q = 0; q < NPT; ++q) {
      const int k = q >> 2, h = q & 3;
      const int x = h == 0 ? v[k].a.x : h == 1 ? v[k].a.z : h == 2 ? v[k].b.x : v[k].b.z;
      const int y = h == 0 ? v[k].a.y : h == 1 ? v[k].a.w : h == 2 ? v[k].b.y : v[k].b.w;
      const uint32_t ux = (uint32_t)x - minx, uy = (uint32_t)y - miny;
      const uint32_t ti = min(uy >> sb, Hc) * Wc1 + min(ux >> sb, Wc);
      c[q] = tiles[ti];
    }
    // phase B: fine pixels of mixed tiles; all gathers of the batch in flight together
#pragma unroll
    for (int q = 0; q < NPT; ++q) {
      if (c[q] >= mixmin) {
        const int k = q >> 2, h = q & 3;
        const int x = h == 0 ? v[k].a.x : h == 1 ? v[k].a.z : h == 2 ? v[k].b.x : v[k].b.z;
        const int y = h == 0 ? v[k].a.y : h == 1 ? v[k].a.w : h == 2 ? v[k].b.y : v[k].b.w;
        const uint32_t fx = ((uint32_t)x - minx) >> s, fy = ((uint32_t)y - miny) >> s;
        const uint32_t fidx = COMPACT ? ((((c[q] & 0x7fffu) << b) | (fy & bm)) << b) | (fx & bm) : fy * W + fx;
        c[q] = classify_fine((int32_t)ld_fine(finep + fidx, pol));
      }
    }
    // now c = 0 (none) | owner + 1 | >= 2^31: boundary / multi-owner record ~c
    uint32_t orc = 0;
#pragma unroll
    for (int q = 0; q < NPT; ++q) orc |= c[q];
    // phase C1: boundary points -> warp queue (one smem atomic per lane that has any), drained 32
    // at a time from the top.  Capacity 160 = < 32 left over + 32 lanes x 4 points.
    static_assert(NPT <= 4, "queue capacity assumes <= 4 points per thread per batch");
    if (__any_sync(0xffffffffu, (int)orc < 0)) {
      uint32_t bnd = 0;
#pragma unroll
      for (int q = 0; q < NPT; ++q) bnd |= (c[q] >> 31) << q;
      if (dreg != nullptr && bnd) {
        // defer to the second kernel: one smem atomic per lane, a 16-B store per point
        const uint32_t nb = __popc(bnd);
        const uint32_t dpos = atomicAdd(&s_dfill, nb);
        const bool fits = dpos + nb <= prm.defer_cap;
        uint32_t d = dpos;
#pragma unroll
        for (int q = 0; q < NPT; ++q)
          if ((bnd >> q) & 1u) {
            const int k = q >> 2, h = q & 3;
            const int x = h == 0 ? v[k].a.x : h == 1 ? v[k].a.z : h == 2 ? v[k].b.x : v[k].b.z;
            const int y = h == 0 ? v[k].a.y : h == 1 ? v[k].a.w : h == 2 ? v[k].b.y : v[k].b.w;
            if (fits) dreg[d] = DEntry{x, y, ~c[q], (uint32_t)prm.head + 4 * (base + k * T + tid) + h};
            else if (d < prm.defer_cap) dreg[d] = DEntry{0, 0, kHole, 0u};   // region full: hole
            ++d;
          }
        if (fits) bnd = 0;                                  // else: fall back to the warp queue
      }
      if (__any_sync(0xffffffffu, bnd != 0u)) {
      if (bnd) {
        int pos = atomicAdd(&s_qn[warp], __popc(bnd));
#pragma unroll
        for (int q = 0; q < NPT; ++q)
          if ((bnd >> q) & 1u) {
            const int k = q >> 2, h = q & 3;
            wq[pos++] = QEntry{~c[q], (uint32_t)prm.head + 4 * (base + k * T + tid) + h};
          }
      }
      __syncwarp();
      int qn = s_qn[warp];
      if (qn >= 32) {
        do {
          drain<MODE>(prm.cvg, prm.xy, wq + qn - 32, 32, lane, myhist, prm.o);
          qn -= 32;
        } while (qn >= 32);
        __syncwarp();
        if (lane == 0) s_qn[warp] = qn;
      }
      __syncwarp();
      }
    }
    // phase C2: direct hits
    if (MODE == kCountSmem) {
      // branch-free: non-hits (0 - 1 = 0xFFFFFFFF, boundary >= 2^31 - 1) go to the trash bin P
#pragma unroll
      for (int q = 0; q < NPT; ++q) atomicAdd(&myhist[min(c[q] - 1u, P)], 1u);
    } else if (MODE == kCountGlobal) {
#pragma unroll
      for (int q = 0; q < NPT; ++q)
        if (c[q] != 0u && !(c[q] >> 31)) atomicAdd(prm.o.counts + (c[q] - 1u), 1ull);
    } else {
      // CTA-aggregated reservation of output slots for this batch (Map with a scan).
      // Within the warp the results are laid out slot-major (all lanes' slot 0 hits, then slot 1,
      // ...), so every store instruction writes one contiguous run: coalesced 8-B / 4-B stores.
      unsigned hm[NPT];
      int wtot = 0;
#pragma unroll
      for (int q = 0; q < NPT; ++q) {
        hm[q] = __ballot_sync(0xffffffffu, c[q] != 0u && !(c[q] >> 31));
        wtot += __popc(hm[q]);
      }
      if (lane == 0) s_scan[warp] = wtot;
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
      int64_t wpos = s_base[warp];
      const unsigned lt = (1u << lane) - 1u;
#pragma unroll
      for (int q = 0; q < NPT; ++q) {
        if ((hm[q] >> lane) & 1u) {
          const int64_t pos = wpos + __popc(hm[q] & lt);
          if (pos < prm.o.cap) {
            const int k = q >> 2, hh = q & 3;
            prm.o.out_ids[pos] = prm.o.id_base + prm.head + 4 * (int64_t)(base + k * T + tid) + hh;
            if (MODE == kPairs) prm.o.out_poly[pos] = (int)c[q] - 1;
          }
        }
        wpos += __popc(hm[q]);
      }
      __syncthreads();   // s_scan / s_base reuse next batch
    }
  }
  __syncwarp();
  if (s_qn[warp] > 0) drain<MODE>(prm.cvg, prm.xy, wq, s_qn[warp], lane, myhist, prm.o);
  if (dreg != nullptr) {
    __syncthreads();
    if (tid == 0) prm.defer_fill[blockIdx.x] = min(s_dfill, prm.defer_cap);
  }
  if (MODE == kCountSmem) {
    __syncthreads();
    for (uint32_t i = tid; i < P; i += T) {
      unsigned long long sum = 0;
#pragma unroll
      for (int k = 0; k < kHC; ++k) sum += hist[k * (P + 1) + i];
      if (sum) atomicAdd(prm.o.counts + i, sum);
    }
  }
}

// Second kernel: the deferred boundary points of every CTA region, one per thread, exact test
// over the pixel's edges (pip_eval).  COUNT: shared-memory histogram (or global atomics);
// SELECT/PAIRS: per-block count pass, block scan, one global atomic, write pass.
template <int MODE>
__global__ void __launch_bounds__(256) k_deferred(const CanvasDev* __restrict__ cvg, const DEntry* __restrict__ defer,
                                                  uint32_t cap, const unsigned int* __restrict__ fill, int nreg, Out o,
                                                  int smem_hist) {
  using BS = cub::BlockScan<int, 256>;
  __shared__ typename BS::TempStorage tmp;
  __shared__ unsigned long long s_gb;
  __shared__ long long s_pre[1025];              // exclusive prefix of the region fills
  extern __shared__ unsigned int dh[];
  const int P = cvg->num_polys;
  const bool sh = MODE == kCountSmem && smem_hist;
  if (sh)
    for (int i = threadIdx.x; i < P; i += 256) dh[i] = 0u;
  if (threadIdx.x == 0) {                        // nreg <= 1024 regions (one per probe CTA)
    long long a = 0;
    for (int r = 0; r < nreg; ++r) { s_pre[r] = a; a += fill[r]; }
    s_pre[nreg] = a;
  }
  __syncthreads();
  const long long total = s_pre[nreg];
  // flattened index space [0, total) in block-sized chunks, grid-stride (all threads loop together)
  for (long long b0 = (long long)blockIdx.x * 256; b0 < total; b0 += (long long)gridDim.x * 256) {
    const long long v = b0 + threadIdx.x;
    DEntry e{0, 0, kHole, 0u};
    if (v < total) {
      int lo = 0, hi = nreg;                     // region r: s_pre[r] <= v < s_pre[r + 1]
      while (hi - lo > 1) { const int mid = (lo + hi) >> 1; if (s_pre[mid] <= v) lo = mid; else hi = mid; }
      e = defer[(size_t)lo * cap + (size_t)(v - s_pre[lo])];
    }
    const bool act = e.rec != kHole;
    const int64_t pid = o.id_base + (int64_t)e.pidx;
    if (MODE == kCountSmem || MODE == kCountGlobal) {
      if (act) pip_eval(cvg, e.x, e.y, e.rec, [&](int q) {
        if (sh) atomicAdd(&dh[q], 1u); else atomicAdd(o.counts + q, 1ull);
      });
    } else {
      int nres = 0;
      if (act) {
        if (MODE == kSelect) { bool any = false; pip_eval(cvg, e.x, e.y, e.rec, [&](int) { any = true; }); nres = any; }
        else pip_eval(cvg, e.x, e.y, e.rec, [&](int) { ++nres; });
      }
      int excl, tot;
      BS(tmp).ExclusiveSum(nres, excl, tot);
      if (threadIdx.x == 0) s_gb = tot ? atomicAdd(o.total, (unsigned long long)tot) : 0ull;
      __syncthreads();
      int64_t pos = (int64_t)s_gb + excl;
      if (nres) {
        if (MODE == kSelect) {
          if (pos < o.cap) o.out_ids[pos] = pid;
        } else {
          pip_eval(cvg, e.x, e.y, e.rec, [&](int q) {
            if (pos < o.cap) { o.out_ids[pos] = pid; o.out_poly[pos] = q; }
            ++pos;
          });
        }
      }
      __syncthreads();
    }
  }
  if (sh) {
    __syncthreads();
    for (int q = threadIdx.x; q < P; q += 256)
      if (dh[q]) atomicAdd(o.counts + q, (unsigned long long)dh[q]);
  }
}

// Stream-ordered scratch comes from the device's default memory pool; by default the pool hands
// memory back to the driver at every synchronisation, which made each call re-map its scratch.
void keep_pool_memory() {
  static bool done = false;
  if (done) return;
  done = true;
  int dev = 0;
  cudaGetDevice(&dev);
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
    uint64_t thr = 16ull << 30;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  cudaGetLastError();
}

bool defer_enabled(int MODE) {
  static const int env = [] { const char* e = getenv("SPADE_DEFER"); return e ? atoi(e) : -1; }();
  if (env >= 0) return env != 0;
  return MODE == kSelect || MODE == kPairs || true;
}

template <int MODE, int T, int U, int PF, int COMPACT>
int launch(const spade_canvas* c, const int2* xy, int64_t n, const Params& base, size_t extra_smem, cudaStream_t st) {
  const size_t smem = tiles_bytes_for(c->d.Wc, c->d.Hc) + (T / 32) * qcap_for(U) * sizeof(QEntry) + extra_smem;
  auto kern = k_probe<MODE, T, U, PF, COMPACT>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return check_cuda(e, "probe smem attribute");
  const int sms = device_sm_count();
  // launches of fewer than 2^31 points (32-bit vector indices and queue point offsets)
  const int64_t kMax = (1ll << 31) - 64;
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
    // deferred boundary regions: n/grid/8 entries per CTA (overflow falls back to in-loop drains)
    DEntry* dbuf = nullptr;
    unsigned int* dfill = nullptr;
    if (defer_enabled(MODE)) {
      keep_pool_memory();
      const int64_t per = std::min<int64_t>(std::max<int64_t>(m / grid / 16, 1024), 1 << 22);
      p.defer_cap = (uint32_t)per;
      if (cudaMallocAsync((void**)&dbuf, sizeof(DEntry) * per * grid, st) != cudaSuccess ||
          cudaMallocAsync((void**)&dfill, sizeof(unsigned int) * grid, st) != cudaSuccess) {
        cudaGetLastError();                       // no scratch: drain in-loop instead
        if (dbuf) cudaFreeAsync(dbuf, st);
        dbuf = nullptr; dfill = nullptr;
      }
      p.defer = dbuf;
      p.defer_fill = dfill;
    }
    kern<<<grid, T, smem, st>>>(p);
    count_launch();
    e = cudaGetLastError();
    if (e != cudaSuccess) return check_cuda(e, "probe launch");
    if (dbuf) {
      const int P = c->d.num_polys;
      const int sh = (MODE == kCountSmem && (size_t)P * 4 <= 96 * 1024) ? 1 : 0;
      const size_t dsm = sh ? (size_t)P * 4 : 0;
      if (dsm > 48 * 1024) cudaFuncSetAttribute(k_deferred<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsm);
      k_deferred<MODE><<<sms * 8, 256, dsm, st>>>(c->d_dev, dbuf, p.defer_cap, dfill, grid, p.o, sh);
      count_launch();
      e = cudaGetLastError();
      cudaFreeAsync(dbuf, st);
      cudaFreeAsync(dfill, st);
      if (e != cudaSuccess) return check_cuda(e, "deferred boundary launch");
    }
  }
  return SPADE_OK;
}

constexpr size_t kSmemBudget = 227 * 1024;

// Launch-shape variants of the probe (threads per CTA, 4-point vectors per thread per batch,
// register double-buffered prefetch of the next batch).  SPADE_PROBE_VARIANT=<i> overrides the
// default for tuning runs; the default is the measured best.
struct Variant { int T, U, PF; };
constexpr Variant kVariants[] = {{1024, 1, 1}, {768, 1, 1}, {512, 1, 1}};
constexpr int kDefaultVariant = 0;

int variant_index() {
  static int v = [] {
    const char* e = getenv("SPADE_PROBE_VARIANT");
    int i = e ? atoi(e) : kDefaultVariant;
    return (i >= 0 && i < (int)(sizeof(kVariants) / sizeof(kVariants[0]))) ? i : kDefaultVariant;
  }();
  return v;
}

template <int MODE, int COMPACT>
int launch_variant2(const spade_canvas* c, const int2* xy, int64_t n, const Params& p, size_t extra, cudaStream_t st) {
  switch (variant_index()) {
    case 1: return launch<MODE, 768, 1, 1, COMPACT>(c, xy, n, p, extra, st);
    case 2: return launch<MODE, 512, 1, 1, COMPACT>(c, xy, n, p, extra, st);
    default: return launch<MODE, 1024, 1, 1, COMPACT>(c, xy, n, p, extra, st);
  }
}

template <int MODE>
int launch_variant(const spade_canvas* c, const int2* xy, int64_t n, const Params& p, size_t extra, cudaStream_t st) {
  return c->d.compact ? launch_variant2<MODE, 1>(c, xy, n, p, extra, st) : launch_variant2<MODE, 0>(c, xy, n, p, extra, st);
}

size_t fixed_smem(const spade_canvas* c) {
  const Variant v = kVariants[variant_index()];
  return tiles_bytes_for(c->d.Wc, c->d.Hc) + (v.T / 32) * qcap_for(v.U) * sizeof(QEntry);
}

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
  const size_t hist = (size_t)kHC * (c->d.num_polys + 1) * 4;
  if (fixed_smem(c) + hist <= kSmemBudget) return launch_variant<kCountSmem>(c, (const int2*)xy, n, p, hist, st);
  return launch_variant<kCountGlobal>(c, (const int2*)xy, n, p, 0, st);
}

int launch_select(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t base, int64_t* out, int64_t cap,
                  unsigned long long* d_total, cudaStream_t st) {
  if (c->empty || n == 0) return SPADE_OK;
  Params p = base_params(c);
  p.o.id_base = base; p.o.out_ids = out; p.o.cap = cap; p.o.total = d_total;
  return launch_variant<kSelect>(c, (const int2*)xy, n, p, 128 * sizeof(int) + 32 * sizeof(long long), st);
}

int launch_pairs(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t base, int64_t* opt, int32_t* opl,
                 int64_t cap, unsigned long long* d_total, cudaStream_t st) {
  if (c->empty || n == 0) return SPADE_OK;
  Params p = base_params(c);
  p.o.id_base = base; p.o.out_ids = opt; p.o.out_poly = opl; p.o.cap = cap; p.o.total = d_total;
  return launch_variant<kPairs>(c, (const int2*)xy, n, p, 128 * sizeof(int) + 32 * sizeof(long long), st);
}

}  // namespace spade
