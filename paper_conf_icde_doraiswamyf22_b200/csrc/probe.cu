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
//   * one persistent 1024-thread CTA per SM; the coarse canvas (<= 80K uint16 tiles + a sentinel
//     column/row) is copied into shared memory once per CTA, so most points are classified by
//     ONE shared-memory load;
//   * points stream with 256-bit loads (LDG.E.256, L1::no_allocate, L2::evict_first), 4 points per
//     thread per batch, and the next batch's loads are issued before the current batch is processed;
//   * points in mixed tiles gather one int32 fine pixel (compact mixed-tile layout, L2 evict_last);
//   * boundary points (a few %) are appended to a per-CTA region in global memory and tested by a
//     second, load-balanced kernel (k_deferred) against the few edges touching their pixel;
//   * COUNT: shared-memory per-polygon histogram (copies selected by lane), flushed once per CTA
//     with 64-bit global atomics; SELECT/PAIRS: CTA-aggregated output reservation (one global
//     atomic per 4096-point batch), slot-major coalesced stores.
#include <cstdint>
#include <climits>
#include <algorithm>
#include <cstdlib>
#include <vector>
#include <cstdio>
#include <atomic>
#include <type_traits>
#include <cub/block/block_scan.cuh>
#include <cub/block/block_radix_sort.cuh>
#include <cub/block/block_reduce.cuh>
#include "spade_internal.cuh"

namespace spade {

namespace {

enum Mode { kCountSmem = 0, kCountGlobal = 1, kSelect = 2, kPairs = 3 };

#ifndef SPADE_PROBE_T
#define SPADE_PROBE_T 1024
#endif
constexpr int kT = SPADE_PROBE_T;  // threads per CTA (one CTA per SM)
constexpr int kNW = kT / 32;
constexpr int kNPT = 4;            // points per thread per batch (one 256-bit vector)
// Shared memory above ~196 KB per CTA shrinks the L1 carve-out below ~60 KB and costs ~35%
// (measured on B200); the histogram copies are chosen to stay under it.
constexpr size_t kSmemSoft = 196 * 1024;
constexpr size_t kSmemL1Step = 164 * 1024;   // the next carve-out step down (L1 60 -> ~92 KB)

struct alignas(32) Vec4 { int4 a, b; };   // 4 points

// Deferred boundary point (the exact test runs in the second kernel).
struct alignas(16) DEntry { int x, y; uint32_t rec, pidx; };
constexpr uint32_t kHole = 0xffffffffu;   // DEntry.rec of a reserved-but-unused slot

// Boundary point in a warp's shared-memory queue (COUNT with an in-loop exact test): just the
// point; the drain re-derives its record from the canvas (shared memory + an L2-resident pixel).
struct alignas(8) QEntry { int x, y; };
constexpr int kQCap = 32 + 32 * kNPT;     // < 32 left over + one batch of the warp's points

__device__ __forceinline__ Vec4 ld_stream(const Vec4* p) {
  Vec4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r.a.x), "=r"(r.a.y), "=r"(r.a.z), "=r"(r.a.w), "=r"(r.b.x), "=r"(r.b.y), "=r"(r.b.z),
                 "=r"(r.b.w)
               : "l"(p));
  return r;
}

// L2 policy of the fine-canvas gathers: evict_last for a fraction `f` of the lines (by address),
// evict_unchanged for the rest (f = 1: every gather evict_last)
__device__ __forceinline__ uint64_t policy_evict_last(float f) {
  uint64_t pol;
  if (f >= 1.0f) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  else asm volatile("createpolicy.fractional.L2::evict_last.L2::evict_unchanged.b64 %0, %1;" : "=l"(pol) : "f"(f));
  return pol;
}
__device__ __forceinline__ uint32_t ld_fine(const int32_t* p, uint64_t pol) {
  uint32_t r;
  asm volatile("ld.global.nc.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
  return r;
}

__device__ __forceinline__ uint32_t ld_fine16(const uint16_t* p, uint64_t pol) {
  uint32_t r;
  asm volatile("ld.global.nc.L2::cache_hint.u16 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
  return r;
}
// class of a 16-bit fine code (spade_internal.cuh kF16*): owner + 1, 0 = none, or ~0 = a record
// (boundary / multi-owner pixel; the record itself is found through the int32 canvas)
__device__ __forceinline__ uint32_t class16(uint32_t code) {
  return code < kF16Empty ? code + 1u : code == kF16Empty ? 0u : 0xffffffffu;
}

// 4-byte asynchronous copy global -> shared (LDGSTS): the gathered value lands in shared memory,
// so the number of gathers in flight is not bounded by registers
__device__ __forceinline__ void cp_async4(uint32_t saddr, const void* g, uint64_t pol) {
  asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 4, %2;" ::"r"(saddr), "l"(g), "l"(pol) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// TMA (bulk async copy) helpers: one mbarrier per warp, 1-D bulk copies global -> shared
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t phase) {
  asm volatile("{\n .reg .pred p;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra WAIT_%=;\n}"
               ::"r"(bar), "r"(phase) : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar, uint64_t pol) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
               ::"r"(dst), "l"(src), "r"(bytes), "r"(bar), "l"(pol) : "memory");
}

__device__ __forceinline__ uint32_t ctaid_x() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%ctaid.x;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t nctaid_x() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%nctaid.x;" : "=r"(r));
  return r;
}

// The record (header blob unit) of point (x, y) on a boundary / multi-owner pixel, from the
// int32 canvas (the fine16 layout's records; rare in-probe paths of any layout).
__device__ __forceinline__ uint32_t rec_of_point(const CanvasDev* __restrict__ cvg, int x, int y) {
  const CanvasDev& cv = *cvg;
  const uint32_t fx = ((uint32_t)x - (uint32_t)cv.minx) >> cv.s, fy = ((uint32_t)y - (uint32_t)cv.miny) >> cv.s;
  return (uint32_t)(-2 - __ldg(cv.fine + ((size_t)fy * (uint32_t)cv.W + fx)));
}

struct U4 {
  uint32_t c[4];
  __device__ __forceinline__ uint32_t& operator[](int i) { return c[i]; }
};

// Output side of a launch (what the sinks write).
// SELECT/PAIRS output slots are handed out in chunks of `chunk` slots per warp (one global atomic
// per chunk, no CTA barrier in the probe loop).  Every warp's last chunk is partly unused: its
// hole is recorded and k_fixup/k_move fill the holes with the results stored past them, so the
// output ends up dense.  Slots at or past the caller's capacity go to an overflow buffer of
// `ovf_cap` >= (number of warps) x chunk slots, enough to hold all results whenever they fit.
struct Out {
  unsigned long long* counts; // COUNT
  unsigned long long* total;  // SELECT/PAIRS: slots handed out (results + holes; may exceed capacity)
  int64_t* out_ids;           // SELECT ids / PAIRS point ids
  int32_t* out_poly;          // PAIRS polygon ids
  int64_t cap;
  int64_t id_base;            // point id of xy[0]
  int64_t* ovf_ids;           // overflow slots [cap, cap + ovf_cap)
  int32_t* ovf_poly;
  int64_t ovf_cap;
  longlong2* holes;           // [grid * kNW] (start, length) of each warp's unused chunk tail
  uint32_t chunk;             // slots per warp chunk
};

template <int MODE>
__device__ __forceinline__ void put_result(const Out& o, int64_t pos, int64_t id, int poly) {
  if (pos < o.cap) {
    // streaming stores (evict-first): the output must not push the canvas out of L2 (measured
    // against default write-back and L2::evict_last stores: C4 5.66 vs 5.73 / 5.92 ms)
    __stcs((long long*)o.out_ids + pos, (long long)id);
    if (MODE == kPairs) __stcs(o.out_poly + pos, poly);
  } else if (pos - o.cap < o.ovf_cap) {
    o.ovf_ids[pos - o.cap] = id;
    if (MODE == kPairs) o.ovf_poly[pos - o.cap] = poly;
  }
}

struct Params {
  CanvasDev cv;
  const CanvasDev* cvg;       // the same, in global memory (for the out-of-line exact test)
  DEntry* defer;              // per-CTA regions of defer_cap entries
  uint32_t defer_cap;
  unsigned int* defer_fill;   // [grid] entries used per CTA region
  uint32_t hcopies;           // COUNT histogram copies in shared memory (power of 2)
  uint32_t cache_slots;       // COUNT with global counts: shared-memory count cache slots (pow 2, or 0)
  uint32_t defer_xy;          // pipelined probe: deferral entries carry the point (re-read from L2)
  float l2_frac;              // fraction of fine-canvas lines gathered with L2::evict_last
  unsigned int* rec_cnt;      // COUNT over overlapping polygons: points per multi-owner record, or null
  uint32_t multi_base;        // blob unit of the first multi-owner record header (records at or past it have no edges)
  uint32_t tma_off;           // QUEUE == 2: byte offset of the TMA stream stages in dynamic shared memory
  unsigned int* kcnt;         // COUNT with K aggregation: points per boundary record, or null
  const int32_t* cfine_tile0;  // compact layout: cfine - (0x8000 << 2b), the block of tile entry 0x8000 (b <= 8)
  const int2* xy;
  int64_t n;
  int64_t head;               // points before the first 32-byte aligned one (0..3)
  int64_t nvec;               // aligned 4-point vectors after the head
  Out o;
};

// COUNT, multi-owner pixels (overlapping polygons, no edge in the pixel): the point's polygons
// are exactly the record's owner set, so the point is counted once per record here and the
// per-record counts are spread over the owner sets after the probe (k_multi_expand) — the
// paper's aggregation plan for points: partial aggregates per canvas location, then combined
// per polygon.  One global atomic per such point instead of one per (point, polygon).
template <int MODE, int LAYOUT = 0, class C>
__device__ __forceinline__ void count_multi_owner(const Params& prm, C& c) {
  // (fine16: a record's id is not in the 16-bit code; the exact-test stage counts them)
  if (!(MODE == kCountSmem || MODE == kCountGlobal) || LAYOUT == 2 || prm.rec_cnt == nullptr) return;
  // (one warp vote on the way in; measured: C3 1.72 -> 1.69 ms against a per-lane test, ov flat.
  // Warp-aggregating the atomics with __match_any_sync was measured too: ov 29.1 -> 29.5-29.9 ms,
  // the lanes of a warp rarely share a record; removing them altogether gives 24.6 ms)
  const unsigned act = __activemask();
  if (!__any_sync(act, (int)(c[0] | c[1] | c[2] | c[3]) < 0)) return;
#pragma unroll
  for (int q = 0; q < kNPT; ++q)
    if ((c[q] >> 31) && ~c[q] >= prm.multi_base) {
      atomicAdd(prm.rec_cnt + (~c[q] - prm.multi_base), 1u);
      c[q] = 0u;
    }
}

// COUNT with global counters, one hit of polygon `key`: the shared-memory count cache (direct
// mapped; the first polygon to claim a slot keeps it for the CTA's lifetime, so hot polygons of
// clustered points claim early), else one global atomic.  Same-slot lanes of a warp serialise in
// the shared-memory atomic unit (cheaper than aggregating them with __match_any_sync first:
// C5 13.6 -> 11.6 ms).
__device__ __forceinline__ void count_cached(uint32_t* ctag, unsigned int* ccnt, uint32_t cslots,
                                             unsigned long long* counts, uint32_t key) {
  if (cslots) {
    const uint32_t sl = key & (cslots - 1u);
    uint32_t t = ctag[sl];
    if (t == 0xffffffffu) { t = atomicCAS(&ctag[sl], 0xffffffffu, key); if (t == 0xffffffffu) t = key; }
    if (t == key) { atomicAdd(&ccnt[sl], 1u); return; }
  }
  atomicAdd(counts + key, 1ull);
}

// Point class after the fine gather: c = fine pixel value + 1, i.e. 0 = no polygon,
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

// Exact test for a point on boundary pixel (or multi-owner pixel) record `rec`:
//   inside(p, P) = [P in K] XOR parity_P(hit over P's primitives touching the pixel),
// the parities of all (<= 64) polygons of the pixel accumulated at once as a bit mask.  A
// primitive's hit: polygon edge -> local_bit (edges that straddle neither y = py nor x = X
// contribute nothing and skip the cross products); disk (KIND == kDisks) ->
// (px-cx)^2 + (py-cy)^2 <= r2 (|px-cx|, |py-cy| < 2^31 for a point on a pixel the disk touches).
// emit(P) is called for every polygon containing the point, in increasing polygon order.
__device__ __forceinline__ bool disk_hit(int4 g, int px, int py) {
  const long long dx = (long long)px - g.x, dy = (long long)py - g.y;
  return (unsigned long long)(dx * dx) + (unsigned long long)(dy * dy) <= (unsigned long long)disk_r2(g);
}

__device__ __forceinline__ int4 ld_prim(const short4* p) { const short4 v = __ldg(p); return make_int4(v.x, v.y, v.z, v.w); }
__device__ __forceinline__ int4 ld_prim(const int4* p) { return __ldg(p); }
__device__ __forceinline__ uint64_t ld_mask(const uint8_t* p) { return __ldg(p); }
__device__ __forceinline__ uint64_t ld_mask(const uint64_t* p) { return __ldg(p); }

// Hit of one primitive for point (px, py) in the pixel whose left side is x = X (the primitive
// and the point in the same coordinates: absolute, or relative to the pixel corner).  An edge that
// straddles neither y = py nor x = X contributes nothing (cr and cu both 0): two compares.
template <int KIND>
__device__ __forceinline__ bool prim_hit(int4 g, int X, int px, int py) {
  if (KIND == kDisks) return disk_hit(g, px, py);
  return (((g.y > py) != (g.w > py)) || ((g.x > X) != (g.z > X))) && local_bit(g, X, px, py);
}

// XOR of the toggle masks of the hit primitives.  U > 1 (the deferred kernel, one point per
// thread): the primitives are loaded U at a time before any is tested, so a record costs
// ~ne / U dependent round trips instead of ne.
template <int KIND, int U, class PT, class MT>
__device__ __forceinline__ uint64_t hit_mask(const PT* __restrict__ seg, const MT* __restrict__ msk, int ne, int X, int px, int py) {
  uint64_t m = 0;
  if (U > 1) {
    // byte masks held in 32-bit registers (the deferred kernel runs at its register limit)
    using MV = typename std::conditional<sizeof(MT) == 1, uint32_t, uint64_t>::type;
    for (int e0 = 0; e0 < ne; e0 += U) {
      int4 g[U];
      MV mk[U];
#pragma unroll
      for (int k = 0; k < U; ++k) {
        const int e = e0 + k < ne ? e0 + k : ne - 1;     // clamped: in bounds, tested once
        g[k] = ld_prim(seg + e);
        mk[k] = (MV)ld_mask(msk + e);
      }
#pragma unroll
      for (int k = 0; k < U; ++k) {
        if (e0 + k >= ne) break;
        if (prim_hit<KIND>(g[k], X, px, py)) m ^= (uint64_t)mk[k];
      }
    }
  } else {
    for (int e = 0; e < ne; ++e)
      if (prim_hit<KIND>(ld_prim(seg + e), X, px, py)) m ^= ld_mask(msk + e);
  }
  return m;
}

// > kMaskPolys polygons: primitives grouped by local polygon index (mask = index)
template <int KIND, class PT, class Fin>
__device__ __forceinline__ void hit_grouped(const PT* __restrict__ seg, const uint64_t* __restrict__ msk, int ne, int X, int px,
                                            int py, const int32_t* __restrict__ rp, Fin&& finalize) {
  int cur = -1, par = 0;
  for (int e = 0; e < ne; ++e) {
    if (!prim_hit<KIND>(ld_prim(seg + e), X, px, py)) continue;
    const int k = (int)__ldg(msk + e);
    if (k != cur) {
      if (cur >= 0 && par) finalize(__ldg(rp + cur), 1);
      cur = k; par = 0;
    }
    par ^= 1;
  }
  if (cur >= 0 && par) finalize(__ldg(rp + cur), 1);
}

// The record's result: [P in K] XOR parity_P, i.e. the term set K merged with the polygons whose
// bit is set in the parity mask m (bit k = the record's k-th polygon, rp[k]); emit(P) ascending.
// finalize(P, par) is also the hook of the > kMaskPolys path.
template <class Emit>
struct TermMerge {
  const int32_t* sets;
  int32_t term;
  int tn, tb, ti;
  Emit& emit;
  __device__ __forceinline__ TermMerge(const CanvasDev* __restrict__ cv, int32_t t, Emit& e) : sets(cv->sets), term(t), tb(0), ti(0), emit(e) {
    if (t >= 0) tn = 1;
    else if (t == kEmpty) tn = 0;
    else { const int2 g = cv->set_rng[-2 - t]; tb = g.x; tn = g.y; }
  }
  __device__ __forceinline__ int at(int i) const { return term >= 0 ? term : sets[tb + i]; }
  __device__ __forceinline__ void operator()(int P, int par) {
    while (ti < tn && at(ti) < P) emit(at(ti++));
    if (ti < tn && at(ti) == P) { par ^= 1; ++ti; }
    if (par) emit(P);
  }
  __device__ __forceinline__ void mask(uint64_t m, const int32_t* __restrict__ rp) {
    while (m) { const int k = __ffsll((long long)m) - 1; m &= m - 1; (*this)(__ldg(rp + k), 1); }
  }
  __device__ __forceinline__ void rest() { while (ti < tn) emit(at(ti++)); }
};

// The record whose header is at blob unit u (the fine canvas value of a boundary / multi-owner
// pixel is -2 - u; spade_internal.cuh "Packed records").  The header load asks L2 to fetch the
// 256-B block around it (L2::256B), so the record's data -- the next loads of the exact test --
// comes in with the same DRAM access instead of one dependent miss per sector.
__device__ __forceinline__ Rec load_rec(const CanvasDev* __restrict__ cv, uint32_t u, uint32_t* id = nullptr) {
  uint4 h;
  asm("ld.global.nc.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(h.x), "=r"(h.y), "=r"(h.z), "=r"(h.w) : "l"(cv->blob + u));
  if (id) *id = h.w;
  return Rec{u + 1u, (int32_t)h.x, (int32_t)h.y, h.z};
}

// Exact test for a point on the boundary (or multi-owner) pixel of record `rec` (packed layout:
// spade_internal.cuh "Packed records"): the header, then the record's polygons, primitives and
// masks from the same contiguous blob.  emit(P) for every polygon containing the point, ascending.
template <int KIND, int U, class Fin>
__device__ __forceinline__ void pip_edges_rec(const CanvasDev* __restrict__ cv, int px, int py, const Rec r, Fin& fin);

template <int KIND, int U = 1, class Emit>
__device__ __forceinline__ void pip_eval_rec(const CanvasDev* __restrict__ cv, int px, int py, const Rec r, Emit&& emit) {
  TermMerge<Emit> fin(cv, r.term, emit);
  pip_edges_rec<KIND, U>(cv, px, py, r, fin);
  fin.rest();
}

// COUNT with K aggregation: the record's term set K is counted once per point in a per-record
// counter (spread over K after the probe, like multi-owner pixels) and only the edge parity is
// evaluated per point: polygon P with odd parity contributes -1 if P is in K (the point leaves
// it) else +1.  Per point O(hit polygons) instead of O(|K|) (overlapping polygon sets).
template <class Emit>
struct DeltaFin {
  const int32_t* sets;
  int32_t term;
  int tb, tn;
  uint64_t kb;                                   // bit k: the record's k-th polygon is in K (<= 64 polygons)
  Emit& emit;
  __device__ __forceinline__ DeltaFin(const CanvasDev* __restrict__ cv, int32_t t, uint64_t kbits, Emit& e)
      : sets(cv->sets), term(t), tb(0), tn(0), kb(kbits), emit(e) {
    if (t < -1) { const int2 g = cv->set_rng[-2 - t]; tb = g.x; tn = g.y; }
  }
  __device__ __forceinline__ bool inK(int P) const {
    if (term >= 0) return P == term;
    int lo = 0, hi = tn;                         // sorted set: lower bound
    while (lo < hi) { const int mid = (lo + hi) >> 1; if (__ldg(sets + tb + mid) < P) lo = mid + 1; else hi = mid; }
    return lo < tn && __ldg(sets + tb + lo) == P;
  }
  __device__ __forceinline__ void operator()(int P, int par) { if (par) emit(P, inK(P) ? -1 : 1); }
  __device__ __forceinline__ void mask(uint64_t m, const int32_t* __restrict__ rp) {
    while (m) { const int k = __ffsll((long long)m) - 1; m &= m - 1; emit(__ldg(rp + k), ((kb >> k) & 1) ? -1 : 1); }
  }
};
template <int KIND, int U = 1, class Emit>
__device__ __forceinline__ void pip_count_delta(const CanvasDev* __restrict__ cv, int px, int py, uint32_t rec, const Rec r,
                                                unsigned int* __restrict__ kcnt, Emit&& emit) {
  if (r.term != kEmpty) atomicAdd(kcnt + rec, 1u);
  DeltaFin<Emit> fin(cv, r.term, __ldg(cv->kbits + rec), emit);
  pip_edges_rec<KIND, U>(cv, px, py, r, fin);
}

template <int KIND, int U, class Fin>
__device__ __forceinline__ void pip_edges_rec(const CanvasDev* __restrict__ cv, int px, int py, const Rec r, Fin& fin) {
  const int ne = r.ecnt;
  if (ne > 0) {
    const int pc = (int)(r.pinfo & kRecPcnt);
    const unsigned char* blob = (const unsigned char*)(cv->blob + r.blob);
    const int32_t* rp = (const int32_t*)blob;
    const unsigned char* eb = blob + ((pc * 4 + 15) & ~15);
    const int X = cv->minx + (int)((((uint32_t)px - (uint32_t)cv->minx) >> cv->s) << cv->s);
    if (KIND == kPolygons && (r.pinfo & kRecShort)) {
      // primitives relative to the pixel corner (X, Y): the point moves with them
      const int Y = cv->miny + (int)((((uint32_t)py - (uint32_t)cv->miny) >> cv->s) << cv->s);
      const short4* seg = (const short4*)eb;
      const unsigned char* mb = eb + (size_t)ne * 8;
      if (pc <= kMaskPolys)
        fin.mask((r.pinfo & kRecByte) ? hit_mask<KIND, U>(seg, (const uint8_t*)mb, ne, 0, px - X, py - Y)
                                      : hit_mask<KIND, U>(seg, (const uint64_t*)mb, ne, 0, px - X, py - Y), rp);
      else
        hit_grouped<KIND>(seg, (const uint64_t*)mb, ne, 0, px - X, py - Y, rp, fin);
    } else {
      const int4* seg = (const int4*)eb;
      const unsigned char* mb = eb + (size_t)ne * 16;
      if (pc <= kMaskPolys)
        fin.mask((r.pinfo & kRecByte) ? hit_mask<KIND, U>(seg, (const uint8_t*)mb, ne, X, px, py)
                                      : hit_mask<KIND, U>(seg, (const uint64_t*)mb, ne, X, px, py), rp);
      else
        hit_grouped<KIND>(seg, (const uint64_t*)mb, ne, X, px, py, rp, fin);
    }
  }
}
template <int KIND, int U = 1, class Emit>
__device__ __forceinline__ void pip_eval(const CanvasDev* __restrict__ cv, int px, int py, uint32_t rec, Emit&& emit) {
  pip_eval_rec<KIND, U>(cv, px, py, load_rec(cv, rec), emit);
}

// Cooperative exact test: the G lanes of a group share one point (same px, py, rec in every lane);
// lane gl tests primitives gl, gl + G, ... and the parity masks are XOR-reduced over the group
// (every lane of the warp must call this).  Returns the group's mask; `big` = the record has more
// than kMaskPolys polygons (the caller then evaluates it serially with pip_eval).
template <int KIND, int G>
__device__ __forceinline__ uint64_t group_mask(const CanvasDev* __restrict__ cv, bool act, int px, int py, const Rec& r, int gl, bool& big) {
  uint64_t m = 0;
  const int pc = (int)(r.pinfo & kRecPcnt);
  big = act && pc > kMaskPolys;
  if (act && !big && r.ecnt > 0) {
    const int ne = r.ecnt;
    const unsigned char* eb = (const unsigned char*)(cv->blob + r.blob) + ((pc * 4 + 15) & ~15);
    const int X = cv->minx + (int)((((uint32_t)px - (uint32_t)cv->minx) >> cv->s) << cv->s);
    if (KIND == kPolygons && (r.pinfo & kRecShort)) {
      const int Y = cv->miny + (int)((((uint32_t)py - (uint32_t)cv->miny) >> cv->s) << cv->s);
      const short4* seg = (const short4*)eb;
      const unsigned char* mb = eb + (size_t)ne * 8;
      const bool by = r.pinfo & kRecByte;
      for (int k = gl; k < ne; k += G)
        if (prim_hit<KIND>(ld_prim(seg + k), 0, px - X, py - Y)) m ^= by ? ld_mask((const uint8_t*)mb + k) : ld_mask((const uint64_t*)mb + k);
    } else {
      const int4* seg = (const int4*)eb;
      const unsigned char* mb = eb + (size_t)ne * 16;
      const bool by = r.pinfo & kRecByte;
      for (int k = gl; k < ne; k += G)
        if (prim_hit<KIND>(ld_prim(seg + k), X, px, py)) m ^= by ? ld_mask((const uint8_t*)mb + k) : ld_mask((const uint64_t*)mb + k);
    }
  }
#pragma unroll
  for (int off = G / 2; off > 0; off >>= 1) m ^= __shfl_xor_sync(0xffffffffu, m, off);
  return m;
}

template <int MODE>
__device__ __forceinline__ void count_hit(unsigned int* hist, uint32_t hstride, unsigned long long* counts, int owner) {
  if (MODE == kCountSmem) atomicAdd(&hist[(uint32_t)owner * hstride], 1u);
  else atomicAdd(counts + owner, 1ull);
}

// Emission from the rare in-kernel paths (deferral region full, unaligned head/tail): per-lane
// atomics.
template <int MODE, int KIND>
__device__ __noinline__ void rare_emit_point(const CanvasDev* __restrict__ cvg, unsigned int* hist, uint32_t hstride, const Out& o,
                                             int x, int y, uint32_t rec, int64_t pid) {
  if (MODE == kCountSmem || MODE == kCountGlobal) {
    pip_eval<KIND>(cvg, x, y, rec, [&](int p) { count_hit<MODE>(hist, hstride, o.counts, p); });
  } else if (MODE == kSelect) {
    bool any = false;
    pip_eval<KIND>(cvg, x, y, rec, [&](int) { any = true; });
    if (any) put_result<MODE>(o, (int64_t)atomicAdd(o.total, 1ull), pid, 0);
  } else {
    pip_eval<KIND>(cvg, x, y, rec, [&](int p) { put_result<MODE>(o, (int64_t)atomicAdd(o.total, 1ull), pid, p); });
  }
}

template <int MODE, int KIND>
__device__ __forceinline__ void emit_point_inl(const CanvasDev* __restrict__ cvg, unsigned int* hist, uint32_t hstride, const Out& o,
                                             int x, int y, uint32_t rec, int64_t pid) {
  if (MODE == kCountSmem || MODE == kCountGlobal) {
    pip_eval<KIND>(cvg, x, y, rec, [&](int p) { count_hit<MODE>(hist, hstride, o.counts, p); });
  } else if (MODE == kSelect) {
    bool any = false;
    pip_eval<KIND>(cvg, x, y, rec, [&](int) { any = true; });
    if (any) put_result<MODE>(o, (int64_t)atomicAdd(o.total, 1ull), pid, 0);
  } else {
    pip_eval<KIND>(cvg, x, y, rec, [&](int p) { put_result<MODE>(o, (int64_t)atomicAdd(o.total, 1ull), pid, p); });
  }
}

template <int MODE>
__device__ __forceinline__ void rare_emit_owner(unsigned int* hist, uint32_t hstride, const Out& o, int owner, int64_t pid) {
  if (MODE == kCountSmem || MODE == kCountGlobal) count_hit<MODE>(hist, hstride, o.counts, owner);
  else put_result<MODE>(o, (int64_t)atomicAdd(o.total, 1ull), pid, owner);
}

// One scalar point (unaligned head / tail): classify synchronously.
template <int MODE, int KIND>
__device__ __noinline__ void scalar_point(const CanvasDev* __restrict__ cvg, const uint16_t* tiles, unsigned int* hist, uint32_t hstride,
                                          const Out& o, int x, int y, int64_t pid) {
  const CanvasDev cv = *cvg;
  const uint32_t ux = (uint32_t)x - (uint32_t)cv.minx, uy = (uint32_t)y - (uint32_t)cv.miny;
  if (ux > cv.extw || uy > cv.exth) return;
  const uint32_t fx = ux >> cv.s, fy = uy >> cv.s;
  uint32_t c = tiles ? tiles[(fy >> cv.b) * (uint32_t)(cv.Wc + 1) + (fx >> cv.b)] : cv.mix_min;   // null: all mixed
  if (c >= cv.mix_min) c = classify_fine(*fine_ptr(cv, c, fx, fy));
  if (c == 0) return;
  if (c & 0x80000000u) rare_emit_point<MODE, KIND>(cvg, hist, hstride, o, x, y, ~c, pid);
  else rare_emit_owner<MODE>(hist, hstride, o, (int)c - 1, pid);
}

// COUNT, in-loop variant: evaluate up to 32 queued boundary points (one per lane).  Out of line:
// the streaming loop keeps a small register footprint.
template <int MODE, int KIND>
__device__ __forceinline__ void drain_point(const CanvasDev* __restrict__ cvg, const uint16_t* tiles, int x, int y,
                                            unsigned int* hist, uint32_t hstride, unsigned long long* counts,
                                            unsigned int* kcnt) {
  const CanvasDev& cv = *cvg;
  const uint32_t fx = ((uint32_t)x - (uint32_t)cv.minx) >> cv.s, fy = ((uint32_t)y - (uint32_t)cv.miny) >> cv.s;
  const uint32_t t = tiles[(fy >> cv.b) * (uint32_t)(cv.Wc + 1) + (fx >> cv.b)];
  const uint32_t c = classify_fine(__ldg(fine_ptr(cv, t, fx, fy)));
  uint32_t rid = 0;
  const Rec r = load_rec(cvg, ~c, &rid);
  if (kcnt)
    pip_count_delta<KIND>(cvg, x, y, rid, r, kcnt, [&](int q, int d) {
      if (MODE == kCountSmem) atomicAdd(&hist[(uint32_t)q * hstride], (unsigned int)d);
      else atomicAdd(counts + q, (unsigned long long)(long long)d);
    });
  else
    pip_eval_rec<KIND>(cvg, x, y, r, [&](int q) { count_hit<MODE>(hist, hstride, counts, q); });
}

template <int MODE, int KIND>
__device__ __noinline__ void drain(const CanvasDev* __restrict__ cvg, const uint16_t* tiles, const QEntry* wq,
                                   int cnt, int lane, unsigned int* hist, uint32_t hstride, unsigned long long* counts,
                                   unsigned int* kcnt) {
  if (lane < cnt) {
    const QEntry e = wq[lane];
    drain_point<MODE, KIND>(cvg, tiles, e.x, e.y, hist, hstride, counts, kcnt);
  }
}

// COUNT drain over a queue of point indices (the TMA variant): the point is re-read (L2)
template <int MODE, int KIND>
__device__ __noinline__ void drain_idx(const CanvasDev* __restrict__ cvg, const uint16_t* tiles, const uint32_t* wqi,
                                       const int2* __restrict__ xy, int cnt, int lane, unsigned int* hist, uint32_t hstride,
                                       unsigned long long* counts, unsigned int* kcnt) {
  if (lane < cnt) {
    const int2 p = __ldg(xy + wqi[lane]);
    drain_point<MODE, KIND>(cvg, tiles, p.x, p.y, hist, hstride, counts, kcnt);
  }
}

// SELECT/PAIRS, in-loop variant: the exact test of one queued boundary point (lane < cnt), by
// its index into the launch's points: (number of results, first polygon).  Out of line.
template <int MODE, int KIND>
__device__ __noinline__ uint2 drain_eval(const CanvasDev* __restrict__ cvg, const uint16_t* tiles,
                                         const int2* __restrict__ xy, uint32_t pidx) {
  const CanvasDev& cv = *cvg;
  const int2 p = __ldg(xy + pidx);
  const uint32_t fx = ((uint32_t)p.x - (uint32_t)cv.minx) >> cv.s, fy = ((uint32_t)p.y - (uint32_t)cv.miny) >> cv.s;
  const uint32_t t = tiles[(fy >> cv.b) * (uint32_t)(cv.Wc + 1) + (fx >> cv.b)];
  const uint32_t c = classify_fine(__ldg(fine_ptr(cv, t, fx, fy)));
  uint32_t n = 0, first = 0;
  if (MODE == kSelect) {
    pip_eval<KIND>(cvg, p.x, p.y, ~c, [&](int) { n = 1; });
  } else {
    pip_eval<KIND>(cvg, p.x, p.y, ~c, [&](int q) { if (n++ == 0) first = (uint32_t)q; });
  }
  return make_uint2(n, first);
}

// Output slots of one warp-wide emission: result k goes to k < room ? b0 + k : b1 + (k - room).
struct Slots {
  long long b0, b1;
  uint32_t room;
  __device__ __forceinline__ long long at(uint32_t k) const { return k < room ? b0 + k : b1 + (long long)(k - room); }
};

// A queued point with more than one result (overlapping polygons): evaluated again, results
// written to slots k, k+1, ...  Out of line (rare).
template <int KIND>
__device__ __noinline__ void emit_multi(const CanvasDev* __restrict__ cvg, const uint16_t* tiles, const int2* __restrict__ xy,
                                        uint32_t pidx, const Out& o, Slots sl, uint32_t k) {
  const CanvasDev& cv = *cvg;
  const int2 p = __ldg(xy + pidx);
  const uint32_t fx = ((uint32_t)p.x - (uint32_t)cv.minx) >> cv.s, fy = ((uint32_t)p.y - (uint32_t)cv.miny) >> cv.s;
  const uint32_t t = tiles[(fy >> cv.b) * (uint32_t)(cv.Wc + 1) + (fx >> cv.b)];
  const uint32_t c = classify_fine(__ldg(fine_ptr(cv, t, fx, fy)));
  pip_eval<KIND>(cvg, p.x, p.y, ~c, [&](int q) { put_result<kPairs>(o, sl.at(k++), o.id_base + pidx, q); });
}

// Per-CTA shared-memory layout (bytes, in order):
//   tiles   (Wc+1) x (Hc+1) uint16 (pitch Wc+1), rounded up to 16 B; the last column and row are
//           always-empty sentinels: tile coordinates are clamped into them (no extent test)
//   COUNT   hcopies x (P + 1) uint32 bins (bin P = "no polygon" trash bin), copy = lane & (hc-1)
//   QUEUE   (in-loop exact test) kNW x kQCap QEntry (COUNT: coordinates) or uint32 (SELECT/
//           PAIRS: point index) per warp: boundary points
__host__ __device__ __forceinline__ size_t queue_bytes(int mode, int queue = 1) {
  return (size_t)kNW * kQCap * (mode == kSelect || mode == kPairs || queue >= 2 ? sizeof(uint32_t) : sizeof(QEntry));
}
__host__ __device__ __forceinline__ size_t tiles_bytes_for(int Wc, int Hc) { return (((size_t)(Wc + 1) * (Hc + 1)) * 2 + 15) & ~(size_t)15; }

// QUEUE: 0 = boundary points deferred to k_deferred, 1 = in-loop warp queues, 2 = in-loop queues
// and the point stream staged by TMA (COUNT only; the A/B variant of the "tma" option), 3 = in-loop
// queues of 4-B point indices (COUNT: frees shared memory for more histogram copies)
template <int MODE, int COMPACT, int QUEUE, int KIND>
__global__ void __launch_bounds__(kT, 1) k_probe(const __grid_constant__ Params prm) {
  extern __shared__ __align__(16) unsigned char smem[];
  const CanvasDev& cv = prm.cv;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int T = kT, NW = kNW, NPT = kNPT;
  constexpr bool TMA = QUEUE == 2;
  constexpr bool IDXQ = QUEUE >= 2;             // COUNT queue of 4-B point indices (the drain re-reads the point)

  const uint32_t tbytes = (uint32_t)tiles_bytes_for(cv.Wc, cv.Hc);
  uint16_t* tiles = (uint16_t*)smem;
  unsigned char* rest = smem + tbytes;
  const uint32_t P = (uint32_t)cv.num_polys;
  unsigned int* hist = (unsigned int*)rest;                       // COUNT
  uint32_t* ctag = (uint32_t*)rest;                               // COUNT (global): cache tags
  unsigned int* ccnt = (unsigned int*)rest + prm.cache_slots;     //                 cache counts
  unsigned int* myhist = hist + (lane & (prm.hcopies - 1));
  __shared__ unsigned int s_dfill;              // deferred entries reserved by this CTA
  __shared__ int s_qn[kNW];                     // QUEUE: per-warp queue fill
  // (the histogram's size rounded up to 16 B: the queue after it holds 8-B entries)
  QEntry* wq = (QEntry*)(rest + (MODE == kCountSmem ? (prm.hcopies * (P + 1) * 4 + 15u) & ~15u : MODE == kCountGlobal ? prm.cache_slots * 8 : 0)) +
               warp * kQCap;
  uint32_t* wqi = (MODE == kCountSmem || MODE == kCountGlobal ? (uint32_t*)wq - warp * kQCap * 2 : (uint32_t*)rest) +
                  warp * kQCap;                                   // SELECT/PAIRS queue, TMA COUNT queue
  if (QUEUE && lane == 0) s_qn[warp] = 0;

  for (uint32_t i = tid; i < tbytes / 16; i += T) ((int4*)tiles)[i] = __ldg((const int4*)cv.coarse + i);
  if (MODE == kCountSmem)
    for (uint32_t i = tid; i < prm.hcopies * (P + 1); i += T) hist[i] = 0u;
  if (MODE == kCountGlobal)
    for (uint32_t i = tid; i < prm.cache_slots; i += T) { ctag[i] = 0xffffffffu; ccnt[i] = 0u; }
  if (tid == 0) s_dfill = 0;
  // TMA stream stage: one 1-KB slice (the warp's 32 vectors of a batch) + one mbarrier per warp
  const uint32_t tma_stage = (uint32_t)__cvta_generic_to_shared(smem) + prm.tma_off + (uint32_t)warp * 1024u;
  const uint32_t tma_bar = (uint32_t)__cvta_generic_to_shared(smem) + prm.tma_off + (uint32_t)NW * 1024u + 8u * warp;
  if (TMA && lane == 0) mbar_init(tma_bar, 1);
  __syncthreads();
  DEntry* const dreg = QUEUE ? nullptr : prm.defer + (size_t)blockIdx.x * prm.defer_cap;
  const uint64_t pol = policy_evict_last(prm.l2_frac);

  // unaligned head and tail (< 8 points): CTA 0, warp 0
  if (blockIdx.x == 0 && warp == 0) {
    const int64_t tail0 = prm.head + 4 * prm.nvec;
    const int64_t ntail = prm.n - tail0;
    if (lane < prm.head) {
      const int2 p = prm.xy[lane];
      scalar_point<MODE, KIND>(prm.cvg, tiles, myhist, prm.hcopies, prm.o, p.x, p.y, prm.o.id_base + lane);
    } else if (lane >= 4 && lane - 4 < ntail) {
      const int64_t i = tail0 + (lane - 4);
      const int2 p = prm.xy[i];
      scalar_point<MODE, KIND>(prm.cvg, tiles, myhist, prm.hcopies, prm.o, p.x, p.y, prm.o.id_base + i);
    }
  }

  const Vec4* vp = (const Vec4*)(prm.xy + prm.head);
  const uint32_t nvec = (uint32_t)prm.nvec;      // sub-launches hold < 2^31 points (launch())
  const uint32_t chunk = (uint32_t)T;
  const uint32_t minx = (uint32_t)cv.minx, miny = (uint32_t)cv.miny;
  const uint32_t sb = (uint32_t)(cv.s + cv.b), s = (uint32_t)cv.s, Wc = (uint32_t)cv.Wc, W = (uint32_t)cv.W;
  const uint32_t Hc = (uint32_t)cv.Hc, Wc1 = Wc + 1u;
  const uint32_t bm = (1u << cv.b) - 1u, mixmin = cv.mix_min;
  const int32_t* __restrict__ finep = COMPACT == 1 ? cv.cfine : cv.fine;
  const uint16_t* __restrict__ f16p = cv.fine16;
  auto load_batch = [&](Vec4& v, uint32_t base) {
    const uint32_t idx = base + tid;
    if (base + chunk <= nvec) v = ld_stream(vp + idx);       // CTA-uniform: full batch
    else if (idx < nvec) v = ld_stream(vp + idx);
    else { v.a = make_int4(INT32_MIN, INT32_MIN, INT32_MIN, INT32_MIN); v.b = v.a; }
  };
  // SELECT/PAIRS: this warp's output chunk [wbase, wbase + K), wused slots used (lane-uniform)
  const uint32_t K = prm.o.chunk;
  long long wbase = 0;
  uint32_t wcap = 0, wused = 0;
  // Slots for `wtot` results of this warp (lane-uniform).  A new chunk covers at most what the
  // warp can still produce from its direct hits (<= 128 per remaining batch), so the last chunk's
  // hole stays small; results beyond that (multi-polygon points) get a chunk of their own size.
  auto reserve = [&](uint32_t wtot, uint32_t later_batches) {
    Slots sl;
    sl.room = wcap - wused;
    sl.b0 = wbase + wused;
    sl.b1 = 0;
    if (wtot > sl.room) {
      const uint32_t need = wtot - sl.room;
      const uint32_t want = max(need, min(K, need + 128u * min(later_batches, 64u)));
      if (lane == 0) sl.b1 = (long long)atomicAdd(prm.o.total, (unsigned long long)want);
      sl.b1 = __shfl_sync(0xffffffffu, sl.b1, 0);
      wbase = sl.b1;
      wcap = want;
      wused = need;
    } else {
      wused += wtot;
    }
    return sl;
  };
  // SELECT/PAIRS drain of 32 queued points (one per lane, lane < cnt)
  auto drain_out = [&](const uint32_t* q, int cnt, uint32_t later_batches) {
    uint2 r = make_uint2(0u, 0u);
    const uint32_t pidx = lane < cnt ? q[lane] : 0u;
    if (lane < cnt) r = drain_eval<MODE, KIND>(prm.cvg, tiles, prm.xy, pidx);
    uint32_t incl = r.x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += t;
    }
    const uint32_t wtot = __shfl_sync(0xffffffffu, incl, 31);
    if (wtot == 0) return;
    const Slots sl = reserve(wtot, later_batches);
    const uint32_t k = incl - r.x;
    if (r.x == 1) put_result<MODE>(prm.o, sl.at(k), prm.o.id_base + pidx, (int)r.y);
    else if (MODE == kPairs && r.x > 1) emit_multi<KIND>(prm.cvg, tiles, prm.xy, pidx, prm.o, sl, k);
  };
  // phases A + B of one batch: c = 0 (none) | owner + 1 | >= 2^31: boundary / multi-owner record ~c
  auto classify = [&](const Vec4 v) {
    U4 f;
    // phase A: coarse (shared memory) lookup, branch-free.  Offsets from the extent origin are
    // unsigned; points left of / below the origin wrap to huge values and, like points right of /
    // above the canvas, clamp into the always-empty sentinel column / row (exact because
    // 2^(s+b) <= 2^30, see canvas_build.cu).  Padding points (INT32_MIN) land there too.
#pragma unroll
    for (int q = 0; q < NPT; ++q) {
      const int x = q == 0 ? v.a.x : q == 1 ? v.a.z : q == 2 ? v.b.x : v.b.z;
      const int y = q == 0 ? v.a.y : q == 1 ? v.a.w : q == 2 ? v.b.y : v.b.w;
      const uint32_t ux = (uint32_t)x - minx, uy = (uint32_t)y - miny;
      f[q] = tiles[min(uy >> sb, Hc) * Wc1 + min(ux >> sb, Wc)];
    }
    // phase B: fine pixels of mixed tiles; all gathers of the batch in flight together
#pragma unroll
    for (int q = 0; q < NPT; ++q) {
      if (f[q] >= mixmin) {
        const int x = q == 0 ? v.a.x : q == 1 ? v.a.z : q == 2 ? v.b.x : v.b.z;
        const int y = q == 0 ? v.a.y : q == 1 ? v.a.w : q == 2 ? v.b.y : v.b.w;
        const uint32_t fx = ((uint32_t)x - minx) >> s, fy = ((uint32_t)y - miny) >> s;
        if (COMPACT == 1) {        // (see the COUNT loop: tile entry's flag bit folded into cfine_tile0)
          const uint32_t fidx = (f[q] * (bm + 1u) + (fy & bm)) * (bm + 1u) + (fx & bm);
          f[q] = classify_fine((int32_t)ld_fine(prm.cfine_tile0 + fidx, pol));
        } else {
          const uint32_t fidx = fy * W + fx;
          f[q] = COMPACT == 2 ? class16(ld_fine16(f16p + fidx, pol)) : classify_fine((int32_t)ld_fine(finep + fidx, pol));
        }
      }
    }
    return f;
  };
  // phase C of one batch: the sinks.  getxy(q): coordinates of point q of this thread.
  auto process = [&](uint32_t base, U4 c, auto getxy) {
    count_multi_owner<MODE, COMPACT>(prm, c);
    const uint32_t orc = c[0] | c[1] | c[2] | c[3];
    if (QUEUE) {
      // phase C1 (COUNT): boundary points -> warp queue (one smem atomic per lane that has any),
      // drained 32 at a time from the top, in the loop: the ALU-heavy exact tests overlap the
      // memory-bound stream of the other warps
      if (__any_sync(0xffffffffu, (int)orc < 0)) {
        uint32_t bnd = 0;
#pragma unroll
        for (int q = 0; q < NPT; ++q) bnd |= (c[q] >> 31) << q;
        if (bnd) {
          int pos = atomicAdd(&s_qn[warp], __popc(bnd));
#pragma unroll
          for (int q = 0; q < NPT; ++q)
            if ((bnd >> q) & 1u) {
              if (MODE == kSelect || MODE == kPairs) {
                wqi[pos++] = (uint32_t)prm.head + 4 * (base + tid) + q;
              } else {
                const int2 p = getxy(q);
                wq[pos++] = QEntry{p.x, p.y};
              }
            }
        }
        __syncwarp();
        int qn = s_qn[warp];
        if (qn >= 32) {
          do {
            if (MODE == kSelect || MODE == kPairs) drain_out(wqi + qn - 32, 32, (nvec - 1 - base) / (nctaid_x() * chunk));
            else drain<MODE, KIND>(prm.cvg, tiles, wq + qn - 32, 32, lane, myhist, prm.hcopies, prm.o.counts, prm.kcnt);
            qn -= 32;
          } while (qn >= 32);
          __syncwarp();
          if (lane == 0) s_qn[warp] = qn;
        }
        __syncwarp();
      }
    } else if ((int)orc < 0) {
      // phase C1: boundary points -> this CTA's deferral region (one smem atomic per lane that has
      // any, a 16-B store per point); if the region is full, test them right here (rare)
      uint32_t bnd = 0;
#pragma unroll
      for (int q = 0; q < NPT; ++q) bnd |= (c[q] >> 31) << q;
      const uint32_t nb = __popc(bnd);
      uint32_t d = atomicAdd(&s_dfill, nb);
      const bool fits = d + nb <= prm.defer_cap;
#pragma unroll
      for (int q = 0; q < NPT; ++q) {
        if ((bnd >> q) & 1u) {
          const int2 p = getxy(q);
          const uint32_t pidx = (uint32_t)prm.head + 4 * (base + tid) + q;
          if (fits) {
            dreg[d] = DEntry{p.x, p.y, ~c[q], pidx};
          } else {
            if (d < prm.defer_cap) dreg[d] = DEntry{0, 0, kHole, 0u};
            rare_emit_point<MODE, KIND>(prm.cvg, myhist, prm.hcopies, prm.o, p.x, p.y,
                                        COMPACT == 2 ? rec_of_point(prm.cvg, p.x, p.y) : ~c[q], prm.o.id_base + pidx);
          }
          ++d;
        }
      }
    }
    // phase C2: direct hits
    if (MODE == kCountSmem) {
      // branch-free: non-hits (0 - 1 = 0xFFFFFFFF, boundary >= 2^31 - 1) go to the trash bin P
#pragma unroll
      for (int q = 0; q < NPT; ++q) atomicAdd(&myhist[min(c[q] - 1u, P) * prm.hcopies], 1u);
    } else if (MODE == kCountGlobal) {
      // too many polygons for a shared-memory histogram: the count cache
#pragma unroll
      for (int q = 0; q < NPT; ++q)
        if (c[q] != 0u && !(c[q] >> 31)) count_cached(ctag, ccnt, prm.cache_slots, prm.o.counts, c[q] - 1u);
    } else {
      // Output slots for this batch (Map with a scan) from the warp's current chunk: a warp
      // scan (ballots), a new chunk (one global atomic, lane 0) when the batch does not fit.
      // Within the warp the results are laid out slot-major (all lanes' slot 0 hits, then slot 1,
      // ...), so every store instruction writes one or two contiguous runs.
      unsigned hm[NPT];
      uint32_t wtot = 0;
#pragma unroll
      for (int q = 0; q < NPT; ++q) {
        hm[q] = __ballot_sync(0xffffffffu, c[q] != 0u && !(c[q] >> 31));
        wtot += __popc(hm[q]);
      }
      if (wtot) {
        const Slots sl = reserve(wtot, (nvec - 1 - base) / (nctaid_x() * chunk));
        const unsigned lt = (1u << lane) - 1u;
        const int64_t id0 = prm.o.id_base + prm.head + 4 * (int64_t)(base + tid);
        if (sl.room >= wtot && sl.b0 + (long long)wtot <= prm.o.cap) {
          // fast path (warp-uniform): the batch fits the current chunk below the capacity
          long long p0 = sl.b0;
#pragma unroll
          for (int q = 0; q < NPT; ++q) {
            if ((hm[q] >> lane) & 1u) {
              const long long pos = p0 + __popc(hm[q] & lt);
              __stcs((long long*)prm.o.out_ids + pos, (long long)(id0 + q));
              if (MODE == kPairs) __stcs(prm.o.out_poly + pos, (int)c[q] - 1);
            }
            p0 += __popc(hm[q]);
          }
        } else {
          uint32_t k0 = 0;
#pragma unroll
          for (int q = 0; q < NPT; ++q) {
            if ((hm[q] >> lane) & 1u) put_result<MODE>(prm.o, sl.at(k0 + __popc(hm[q] & lt)), id0 + q, (int)c[q] - 1);
            k0 += __popc(hm[q]);
          }
        }
      }
    }
  };
  const uint32_t first = blockIdx.x * chunk;
  if (MODE == kCountSmem || MODE == kCountGlobal) {
    // COUNT (in-loop exact tests: the C3 configuration; or deferred: C5): written out without the
    // lambdas, which cost these register-bound variants a spill of the loop state
    const uint32_t hist_s = (uint32_t)__cvta_generic_to_shared(myhist), hstride_b = 4u * prm.hcopies;
    Vec4 nxt;
    uint32_t tma_phase = 0;
    uint64_t spol = 0;
    if (TMA) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(spol));
    // TMA: lane 0 starts the bulk copy of the warp's slice of the batch at `b0` into its stage
    auto tma_issue = [&](uint32_t b0) {
      const uint32_t w0 = b0 + (uint32_t)warp * 32u;
      if (lane == 0 && w0 < nvec) {
        const uint32_t bytes = min(32u, nvec - w0) * 32u;
        mbar_expect_tx(tma_bar, bytes);
        bulk_g2s(tma_stage, vp + w0, bytes, tma_bar, spol);
      }
    };
    if (TMA) tma_issue(blockIdx.x * chunk);
    else if (blockIdx.x * chunk < nvec) load_batch(nxt, blockIdx.x * chunk);
    // (the stride is re-read from the special register each batch: kept live, it spilled)
#ifdef SPADE_COUNT_UNROLL2
#pragma unroll 2
#endif
    for (uint32_t base = blockIdx.x * chunk; base < nvec; base += nctaid_x() * chunk) {
      Vec4 v;
      const uint32_t stride = nctaid_x() * chunk;
      if (TMA) {
        // wait for this warp's slice, read it from shared memory, start the next batch's copy
        const uint32_t w0 = base + (uint32_t)warp * 32u;
        v.a = make_int4(INT32_MIN, INT32_MIN, INT32_MIN, INT32_MIN); v.b = v.a;
        if (w0 < nvec) {
          mbar_wait(tma_bar, tma_phase);
          tma_phase ^= 1u;
          if (w0 + lane < nvec) {
            const uint32_t a = tma_stage + 32u * lane;
            asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(v.a.x), "=r"(v.a.y), "=r"(v.a.z), "=r"(v.a.w) : "r"(a) : "memory");
            asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(v.b.x), "=r"(v.b.y), "=r"(v.b.z), "=r"(v.b.w) : "r"(a + 16u) : "memory");
          }
        }
        __syncwarp();
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic reads before the async-proxy overwrite
        tma_issue(base + stride);
      } else {
        v = nxt;
        if (base + stride < nvec) load_batch(nxt, base + stride);   // next batch in flight meanwhile
      }
      // phase A: coarse (shared memory) lookup, branch-free.  Offsets from the extent origin are
      // unsigned; points left of / below the origin wrap to huge values and, like points right of /
      // above the canvas, clamp into the always-empty sentinel column / row (exact because
      // 2^(s+b) <= 2^30, see canvas_build.cu).  Padding points (INT32_MIN) land there too.
      uint32_t c[NPT];
#pragma unroll
      for (int q = 0; q < NPT; ++q) {
        const int x = q == 0 ? v.a.x : q == 1 ? v.a.z : q == 2 ? v.b.x : v.b.z;
        const int y = q == 0 ? v.a.y : q == 1 ? v.a.w : q == 2 ? v.b.y : v.b.w;
        const uint32_t ux = (uint32_t)x - minx, uy = (uint32_t)y - miny;
        c[q] = tiles[min(uy >> sb, Hc) * Wc1 + min(ux >> sb, Wc)];
      }
      // phase B: fine pixels of mixed tiles; all gathers of the batch in flight together.
      // Compact layout: the pixel is ((t·B + ly)·B + lx) past cfine_tile0, the base of the block of
      // tile entry t = 0x8000 | m (t's flag bit folded into the base pointer, B = 2^b): two IMADs
      // instead of the shift/mask chain (this phase's instructions issue for every point of a warp
      // in which any point needs a gather, i.e. nearly always).
#pragma unroll
      for (int q = 0; q < NPT; ++q) {
        if (c[q] >= mixmin) {
          const int x = q == 0 ? v.a.x : q == 1 ? v.a.z : q == 2 ? v.b.x : v.b.z;
          const int y = q == 0 ? v.a.y : q == 1 ? v.a.w : q == 2 ? v.b.y : v.b.w;
          const uint32_t fx = ((uint32_t)x - minx) >> s, fy = ((uint32_t)y - miny) >> s;
          if (COMPACT == 1) {
            const uint32_t fidx = (c[q] * (bm + 1u) + (fy & bm)) * (bm + 1u) + (fx & bm);
            c[q] = classify_fine((int32_t)ld_fine(prm.cfine_tile0 + fidx, pol));
          } else {
            const uint32_t fidx = fy * W + fx;
            c[q] = COMPACT == 2 ? class16(ld_fine16(f16p + fidx, pol)) : classify_fine((int32_t)ld_fine(finep + fidx, pol));
          }
        }
      }
      // now c = 0 (none) | owner + 1 | >= 2^31: boundary / multi-owner record ~c
      count_multi_owner<MODE, COMPACT>(prm, c);
      const uint32_t orc = c[0] | c[1] | c[2] | c[3];
      if (!QUEUE) {
        // phase C1 (COUNT, deferred): boundary points -> this CTA's deferral region (one smem
        // atomic per lane that has any, a 16-B store per point); region full: tested right here
        if ((int)orc < 0) {
          uint32_t bnd = 0;
#pragma unroll
          for (int q = 0; q < NPT; ++q) bnd |= (c[q] >> 31) << q;
          const uint32_t nb = __popc(bnd);
          uint32_t d = atomicAdd(&s_dfill, nb);
          const bool fits = d + nb <= prm.defer_cap;
#pragma unroll
          for (int q = 0; q < NPT; ++q) {
            if ((bnd >> q) & 1u) {
              const int x = q == 0 ? v.a.x : q == 1 ? v.a.z : q == 2 ? v.b.x : v.b.z;
              const int y = q == 0 ? v.a.y : q == 1 ? v.a.w : q == 2 ? v.b.y : v.b.w;
              // (the region's address is re-derived here: kept live, it spilled)
              DEntry* const dr = prm.defer + (size_t)ctaid_x() * prm.defer_cap;
              if (fits) {
                dr[d] = DEntry{x, y, ~c[q], 0u};
              } else {
                if (d < prm.defer_cap) dr[d] = DEntry{0, 0, kHole, 0u};
                emit_point_inl<MODE, KIND>(prm.cvg, myhist, prm.hcopies, prm.o, x, y,
                                           COMPACT == 2 ? rec_of_point(prm.cvg, x, y) : ~c[q], 0);
              }
              ++d;
            }
          }
        }
      } else {
        // phase C1 (COUNT): boundary points -> warp queue (one smem atomic per lane that has any),
        // drained 32 at a time from the top, in the loop: the ALU-heavy exact tests overlap the
        // memory-bound stream of the other warps
        if (__any_sync(0xffffffffu, (int)orc < 0)) {
          uint32_t bnd = 0;
#pragma unroll
          for (int q = 0; q < NPT; ++q) bnd |= (c[q] >> 31) << q;
          if (bnd) {
            int pos = atomicAdd(&s_qn[warp], __popc(bnd));
#pragma unroll
            for (int q = 0; q < NPT; ++q)
              if ((bnd >> q) & 1u) {
                if (IDXQ) {                  // (index queue: 4-B point indices; the drain re-reads the point)
                  wqi[pos++] = (uint32_t)prm.head + 4 * (base + tid) + q;
                } else {
                  const int x = q == 0 ? v.a.x : q == 1 ? v.a.z : q == 2 ? v.b.x : v.b.z;
                  const int y = q == 0 ? v.a.y : q == 1 ? v.a.w : q == 2 ? v.b.y : v.b.w;
                  wq[pos++] = QEntry{x, y};
                }
              }
          }
          __syncwarp();
          int qn = s_qn[warp];
          if (qn >= 32) {
            do {
              if (IDXQ) drain_idx<MODE, KIND>(prm.cvg, tiles, wqi + qn - 32, prm.xy, 32, lane, myhist, prm.hcopies, prm.o.counts, prm.kcnt);
              else drain<MODE, KIND>(prm.cvg, tiles, wq + qn - 32, 32, lane, myhist, prm.hcopies, prm.o.counts, prm.kcnt);
              qn -= 32;
            } while (qn >= 32);
            __syncwarp();
            if (lane == 0) s_qn[warp] = qn;
          }
          __syncwarp();
        }
      }
      if (MODE == kCountSmem) {
        // phase C2: direct hits (branch-free: non-hits and boundary points go to the trash bin P)
#pragma unroll
        for (int q = 0; q < NPT; ++q)       // one IMAD per address: bin * (4 * copies) + this lane's copy
          asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(min(c[q] - 1u, P) * hstride_b + hist_s) : "memory");
      } else {
        // phase C2, too many polygons for a shared-memory histogram: the count cache
#pragma unroll
        for (int q = 0; q < NPT; ++q)
          if (c[q] != 0u && !(c[q] >> 31)) count_cached(ctag, ccnt, prm.cache_slots, prm.o.counts, c[q] - 1u);
      }
    }
  } else {
    // only the next batch of points is prefetched; there are no CTA barriers in the loop, the 32
    // warps hide each other's gather latency
    Vec4 nxt;
    if (first < nvec) load_batch(nxt, first);
    for (uint32_t base = first; base < nvec; base += nctaid_x() * chunk) {
      const Vec4 v = nxt;
      const uint32_t stride = nctaid_x() * chunk;
      if (base + stride < nvec) load_batch(nxt, base + stride);   // next batch in flight meanwhile
      process(base, classify(v), [v](int q) {
        return make_int2(q == 0 ? v.a.x : q == 1 ? v.a.z : q == 2 ? v.b.x : v.b.z,
                         q == 0 ? v.a.y : q == 1 ? v.a.w : q == 2 ? v.b.y : v.b.w);
      });
    }
  }
  if (MODE == kSelect || MODE == kPairs) {
    if (QUEUE) {
      __syncwarp();
      if (s_qn[warp] > 0) drain_out(wqi, s_qn[warp], 0u);
    }
    if (lane == 0) prm.o.holes[(size_t)blockIdx.x * kNW + warp] = make_longlong2(wbase + wused, (long long)(wcap - wused));
  }
  if (QUEUE && (MODE == kCountSmem || MODE == kCountGlobal)) {
    __syncwarp();
    if (s_qn[warp] > 0) {
      if (IDXQ) drain_idx<MODE, KIND>(prm.cvg, tiles, wqi, prm.xy, s_qn[warp], lane, myhist, prm.hcopies, prm.o.counts, prm.kcnt);
      else drain<MODE, KIND>(prm.cvg, tiles, wq, s_qn[warp], lane, myhist, prm.hcopies, prm.o.counts, prm.kcnt);
    }
  }
  __syncthreads();
  if (!QUEUE && tid == 0) prm.defer_fill[blockIdx.x] = min(s_dfill, prm.defer_cap);
  if (MODE == kCountGlobal)
    for (uint32_t i = tid; i < prm.cache_slots; i += T)
      if (ccnt[i]) atomicAdd(prm.o.counts + ctag[i], (unsigned long long)ccnt[i]);
  if (MODE == kCountSmem) {
    for (uint32_t i = tid; i < P; i += T) {
      unsigned long long sum = 0;
      for (uint32_t k = 0; k < prm.hcopies; ++k) sum += (unsigned long long)(long long)(int)hist[i * prm.hcopies + k];
      if (sum) atomicAdd(prm.o.counts + i, sum);
    }
  }
}

// COUNT probe for canvases whose points mostly need the fine gather (many mixed tiles: C5's 40k
// polygons, the 100K-disk canvases).  The fine pixels are gathered with cp.async into a per-thread
// shared-memory ring of kPipeD batches, so each thread keeps kPipeD x 4 gathers in flight (the
// register-staged probe holds 4); batch j is classified and counted kPipeD - 1 batches after its
// gathers were issued.  Boundary points go to the deferral regions as (record, point index); the
// deferred kernel re-reads their coordinates.
#ifndef SPADE_PIPE_D
#define SPADE_PIPE_D 4
#endif
#ifndef SPADE_PIPE_SMEM_KB
#define SPADE_PIPE_SMEM_KB 196
#endif
constexpr int kPipeD = SPADE_PIPE_D;
constexpr size_t kPipeSmem = (size_t)SPADE_PIPE_SMEM_KB * 1024;
__host__ __device__ __forceinline__ size_t pipe_ring_bytes(int d = kPipeD) { return (size_t)d * kNPT * kT * 4; }
// VAR 2 of the pipelined probe: canvases whose coarse tiles are ALL mixed (C5's 40k polygons)
// skip the tile grid (an extent test instead of the sentinel lookup) and use the shared memory it
// and two ring stages free for a full per-polygon histogram (no count cache, no global atomics)
constexpr int kPipeNoTileD = 2;

template <int MODE, int COMPACT, int KIND, int VAR = 1>
__global__ void __launch_bounds__(kT, 1) k_probe_pipe(const __grid_constant__ Params prm) {
  extern __shared__ __align__(16) unsigned char smem[];
  const CanvasDev& cv = prm.cv;
  const int tid = threadIdx.x, lane = tid & 31;
  constexpr bool NOTILE = VAR == 2;
  constexpr int T = kT, NPT = kNPT, D = NOTILE ? kPipeNoTileD : kPipeD;
  const uint32_t tbytes = NOTILE ? 0u : (uint32_t)tiles_bytes_for(cv.Wc, cv.Hc);
  uint16_t* tiles = (uint16_t*)smem;
  unsigned char* rest = smem + tbytes;
  const uint32_t P = (uint32_t)cv.num_polys;
  unsigned int* hist = (unsigned int*)rest;                       // COUNT (shared memory)
  uint32_t* ctag = (uint32_t*)rest;                               // COUNT (global): cache tags
  unsigned int* ccnt = (unsigned int*)rest + prm.cache_slots;     //                 cache counts
  unsigned int* myhist = hist + (lane & (prm.hcopies - 1));
  const size_t sink_bytes = MODE == kCountSmem ? (size_t)prm.hcopies * (P + 1) * 4 : (size_t)prm.cache_slots * 8;
  int32_t* ring = (int32_t*)(rest + ((sink_bytes + 15) & ~(size_t)15));   // [D][NPT][T] pixel values
  __shared__ unsigned int s_dfill;

  if constexpr (!NOTILE)
    for (uint32_t i = tid; i < tbytes / 16; i += T) ((int4*)tiles)[i] = __ldg((const int4*)cv.coarse + i);
  if (MODE == kCountSmem)
    for (uint32_t i = tid; i < prm.hcopies * (P + 1); i += T) hist[i] = 0u;
  if (MODE == kCountGlobal)
    for (uint32_t i = tid; i < prm.cache_slots; i += T) { ctag[i] = 0xffffffffu; ccnt[i] = 0u; }
  if (tid == 0) s_dfill = 0;
  __syncthreads();
  const uint64_t pol = policy_evict_last(prm.l2_frac);

  if (blockIdx.x == 0 && tid < 32) {               // unaligned head and tail (< 8 points)
    const int64_t tail0 = prm.head + 4 * prm.nvec;
    const int64_t ntail = prm.n - tail0;
    if (lane < prm.head) {
      const int2 p = prm.xy[lane];
      scalar_point<MODE, KIND>(prm.cvg, NOTILE ? nullptr : tiles, myhist, prm.hcopies, prm.o, p.x, p.y, prm.o.id_base + lane);
    } else if (lane >= 4 && lane - 4 < ntail) {
      const int64_t i = tail0 + (lane - 4);
      const int2 p = prm.xy[i];
      scalar_point<MODE, KIND>(prm.cvg, NOTILE ? nullptr : tiles, myhist, prm.hcopies, prm.o, p.x, p.y, prm.o.id_base + i);
    }
  }

  const Vec4* vp = (const Vec4*)(prm.xy + prm.head);
  const uint32_t nvec = (uint32_t)prm.nvec;
  const uint32_t extw = cv.extw, exth = cv.exth;
  const uint32_t minx = (uint32_t)cv.minx, miny = (uint32_t)cv.miny;
  const uint32_t sb = (uint32_t)(cv.s + cv.b), s = (uint32_t)cv.s, Wc = (uint32_t)cv.Wc, W = (uint32_t)cv.W;
  const uint32_t Hc = (uint32_t)cv.Hc, Wc1 = Wc + 1u;
  const uint32_t b = (uint32_t)cv.b, bm = (1u << cv.b) - 1u, mixmin = cv.mix_min;
  const int32_t* __restrict__ finep = COMPACT == 1 ? cv.cfine : cv.fine;
  const uint16_t* __restrict__ f16p = cv.fine16;
  uint32_t halves = 0;                             // fine16: which half of the gathered word, per (batch % D, q)
  const uint32_t first = blockIdx.x * T, stride = nctaid_x() * T;
  const uint32_t nb = first < nvec ? (nvec - first + stride - 1) / stride : 0u;   // batches of this CTA
  const uint32_t ring_s = (uint32_t)__cvta_generic_to_shared(ring) + 4u * tid;
  const uint32_t cslots = prm.cache_slots;
  Vec4 nxt;
  if (nb) {
    if (first + tid < nvec) nxt = ld_stream(vp + first + tid);
    else { nxt.a = make_int4(INT32_MIN, INT32_MIN, INT32_MIN, INT32_MIN); nxt.b = nxt.a; }
  }
  for (uint32_t it = 0; it + 1 < nb + D; ++it) {
    if (it < nb) {
      // issue batch `it`: coarse lookup, fine gathers (or the uniform tile's value) into the ring
      const Vec4 v = nxt;
      const uint32_t nbase = first + (it + 1) * stride;
      if (it + 1 < nb) {
        if (nbase + tid < nvec) nxt = ld_stream(vp + nbase + tid);
        else { nxt.a = make_int4(INT32_MIN, INT32_MIN, INT32_MIN, INT32_MIN); nxt.b = nxt.a; }
      }
      const uint32_t slot = ring_s + (it % D) * (NPT * T * 4);
#pragma unroll
      for (int q = 0; q < NPT; ++q) {
        const int x = q == 0 ? v.a.x : q == 1 ? v.a.z : q == 2 ? v.b.x : v.b.z;
        const int y = q == 0 ? v.a.y : q == 1 ? v.a.w : q == 2 ? v.b.y : v.b.w;
        const uint32_t ux = (uint32_t)x - minx, uy = (uint32_t)y - miny;
        // (NOTILE: every tile is mixed; points outside the extent are empty)
        const uint32_t c = NOTILE ? (ux > extw || uy > exth ? 0u : mixmin) : tiles[min(uy >> sb, Hc) * Wc1 + min(ux >> sb, Wc)];
        const uint32_t sa = slot + q * (T * 4);
        if (c >= mixmin) {
          const uint32_t fx = ux >> s, fy = uy >> s;
          const uint32_t fidx = COMPACT == 1 ? ((((c & 0x7fffu) << b) | (fy & bm)) << b) | (fx & bm) : fy * W + fx;
          if (COMPACT == 2) {
            // cp.async moves >= 4 bytes: the aligned word holding the code, half noted
            const uint32_t hb = (it % D) * NPT + q;
            halves = (halves & ~(1u << hb)) | ((fidx & 1u) << hb);
            cp_async4(sa, f16p + (fidx & ~1u), pol);
          } else {
            cp_async4(sa, finep + fidx, pol);
          }
        } else if (COMPACT == 2) {
          const uint32_t code = c == 0u ? (uint32_t)kF16Empty : c - 1u;    // uniform tile: both halves
          asm volatile("st.shared.b32 [%0], %1;" ::"r"(sa), "r"(code | (code << 16)) : "memory");
        } else {
          asm volatile("st.shared.b32 [%0], %1;" ::"r"(sa), "r"(c - 1u) : "memory");   // pixel value: owner / -1
        }
      }
    }
    cp_async_commit();                               // (an empty group past the last batch)
    if (it + 1 >= D) {
      // consume batch j = it - (D - 1): its gathers are complete
      cp_async_wait<D - 1>();
      const uint32_t j = it + 1 - D;
      const uint32_t slot = ring_s + (j % D) * (NPT * T * 4);
      uint32_t c[NPT];
#pragma unroll
      for (int q = 0; q < NPT; ++q) {
        uint32_t v;
        asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(slot + q * (T * 4)) : "memory");
        if (COMPACT == 2) c[q] = class16((v >> (((halves >> ((j % D) * NPT + q)) & 1u) * 16)) & 0xffffu);
        else c[q] = v + 1u;                          // 0 none | owner + 1 | >= 2^31 record ~c
      }
      count_multi_owner<MODE, COMPACT>(prm, c);
      const uint32_t orc = c[0] | c[1] | c[2] | c[3];
      if ((int)orc < 0) {
        uint32_t bnd = 0;
#pragma unroll
        for (int q = 0; q < NPT; ++q) bnd |= (c[q] >> 31) << q;
        const uint32_t nbd = __popc(bnd);
        uint32_t d = atomicAdd(&s_dfill, nbd);
        const bool fits = d + nbd <= prm.defer_cap;
        DEntry* const dr = prm.defer + (size_t)ctaid_x() * prm.defer_cap;
        const uint32_t pbase = (uint32_t)prm.head + 4u * (first + j * stride + tid);
        // the batch was streamed D - 1 batches ago (evict-first): its points are still in L2, so
        // the entry carries them and k_deferred does not re-read them from DRAM
#pragma unroll
        for (int q = 0; q < NPT; ++q) {
          if ((bnd >> q) & 1u) {
            if (fits) {
              const int2 pt = prm.defer_xy ? __ldcg(prm.xy + pbase + q) : make_int2(0, 0);
              dr[d] = DEntry{pt.x, pt.y, ~c[q], pbase + q};
            } else {
              if (d < prm.defer_cap) dr[d] = DEntry{0, 0, kHole, 0u};
              const int2 p = __ldg(prm.xy + pbase + q);
              emit_point_inl<MODE, KIND>(prm.cvg, myhist, prm.hcopies, prm.o, p.x, p.y,
                                         COMPACT == 2 ? rec_of_point(prm.cvg, p.x, p.y) : ~c[q], 0);
            }
            ++d;
          }
        }
      }
      if (MODE == kCountSmem) {
#pragma unroll
        for (int q = 0; q < NPT; ++q) atomicAdd(&myhist[min(c[q] - 1u, P) * prm.hcopies], 1u);
      } else {
#pragma unroll
        for (int q = 0; q < NPT; ++q)
          if (c[q] != 0u && !(c[q] >> 31)) count_cached(ctag, ccnt, cslots, prm.o.counts, c[q] - 1u);
      }
    }
  }
  cp_async_wait<0>();
  __syncthreads();
  if (tid == 0) prm.defer_fill[blockIdx.x] = min(s_dfill, prm.defer_cap);
  if (MODE == kCountGlobal)
    for (uint32_t i = tid; i < prm.cache_slots; i += T)
      if (ccnt[i]) atomicAdd(prm.o.counts + ctag[i], (unsigned long long)ccnt[i]);
  if (MODE == kCountSmem) {
    for (uint32_t i = tid; i < P; i += T) {
      unsigned long long sum = 0;
      for (uint32_t k = 0; k < prm.hcopies; ++k) sum += (unsigned long long)(long long)(int)hist[i * prm.hcopies + k];
      if (sum) atomicAdd(prm.o.counts + i, sum);
    }
  }
}

// COUNT's second kernel, cooperative: the deferred boundary points of every CTA region, flattened;
// each group of G lanes tests one point (group_mask), its first lane merges the result and counts
// it (shared-memory histogram when the P bins fit, else warp-aggregated global atomics).
template <int MODE, int KIND, int G, int PIX>
__global__ void __launch_bounds__(1024, 1) k_deferred_count(const CanvasDev* __restrict__ cvg, const DEntry* __restrict__ defer,
                                                            uint32_t cap, const unsigned int* __restrict__ fill, int nreg,
                                                            unsigned long long* __restrict__ counts, int smem_hist,
                                                            const int2* __restrict__ pxy) {
  constexpr int T = 1024, GPB = T / G;
  __shared__ long long s_pre[1025];              // exclusive prefix of the region fills
  extern __shared__ unsigned int dh[];
  const int P = cvg->num_polys;
  const int lane = threadIdx.x & 31, gl = lane & (G - 1), grp = threadIdx.x / G;
  if (smem_hist)
    for (int i = threadIdx.x; i < P; i += T) dh[i] = 0u;
  if (threadIdx.x == 0) {                        // nreg <= 1024 regions (one per probe CTA)
    long long a = 0;
    for (int r = 0; r < nreg; ++r) { s_pre[r] = a; a += fill[r]; }
    s_pre[nreg] = a;
  }
  __syncthreads();
  const long long total = s_pre[nreg];
  auto fetch = [&](long long v) {                // entry v of the flattened regions (or a hole)
    DEntry d{0, 0, kHole, 0u};
    if (v < total) {
      int lo = 0, hi = nreg;
      while (hi - lo > 1) { const int mid = (lo + hi) >> 1; if (s_pre[mid] <= v) lo = mid; else hi = mid; }
      d = defer[(size_t)lo * cap + (size_t)(v - s_pre[lo])];
    }
    return d;
  };
  const long long gstride = (long long)gridDim.x * GPB;
  DEntry nxt = fetch((long long)blockIdx.x * GPB + grp);
  for (long long b0 = (long long)blockIdx.x * GPB; b0 < total; b0 += gstride) {   // warp-uniform bound
    DEntry e = nxt;
    nxt = fetch(b0 + gstride + grp);             // the group's next point in flight meanwhile
    const bool act = e.rec != kHole;
    if (act && pxy) { const int2 q = __ldg(pxy + e.pidx); e.x = q.x; e.y = q.y; }   // entry without coordinates
    if (act && PIX) e.rec = rec_of_point(cvg, e.x, e.y);                         // fine16 canvas
    Rec r{0u, kEmpty, 0, 0u};
    if (act) r = load_rec(cvg, e.rec);
    bool big;
    const uint64_t m = group_mask<KIND, G>(cvg, act, e.x, e.y, r, gl, big);
    int first = -1;
    if (act && gl == 0) {
      auto emit = [&](int q) {
        if (smem_hist) atomicAdd(&dh[q], 1u);
        else if (first < 0) first = q;
        else atomicAdd(counts + q, 1ull);
      };
      if (big) {
        pip_eval<KIND>(cvg, e.x, e.y, e.rec, emit);
      } else {
        TermMerge<decltype(emit)> fin(cvg, r.term, emit);
        fin.mask(m, (const int32_t*)(cvg->blob + r.blob));
        fin.rest();
      }
    }
    if (!smem_hist) {                            // each point's first result aggregated over the warp
      const unsigned mm = __match_any_sync(0xffffffffu, first);
      if (first >= 0 && (mm & ((1u << lane) - 1u)) == 0u) atomicAdd(counts + first, (unsigned long long)__popc(mm));
    }
  }
  if (smem_hist) {
    __syncthreads();
    for (int q = threadIdx.x; q < P; q += T)
      if (dh[q]) atomicAdd(counts + q, (unsigned long long)dh[q]);
  }
}

// Second kernel: the deferred boundary points of every CTA region, flattened and spread over
// many blocks (one point per thread), exact test over the pixel's edges (pip_eval).  COUNT:
// shared-memory histogram (or global atomics); SELECT/PAIRS: per-block count pass, block scan,
// one global atomic, write pass.
template <int MODE, int KIND, int PIX, int KAGG>
__global__ void __launch_bounds__(256, 4) k_deferred(const CanvasDev* __restrict__ cvg, const DEntry* __restrict__ defer,
                                                  uint32_t cap, const unsigned int* __restrict__ fill, int nreg, Out o,
                                                  int smem_hist, const int2* __restrict__ pxy, unsigned int* __restrict__ kcnt) {
  using BS = cub::BlockScan<int, 256>;
  __shared__ typename BS::TempStorage tmp;
  __shared__ unsigned long long s_gb;
  __shared__ long long s_pre[1025];              // exclusive prefix of the region fills
  extern __shared__ unsigned int dh[];
  const int P = cvg->num_polys;
  const bool sh = (MODE == kCountSmem || MODE == kCountGlobal) && smem_hist;
  if (sh)
    for (int i = threadIdx.x; i < P; i += 256) dh[i] = 0u;
  if (threadIdx.x == 0) {                        // nreg <= 1024 regions (one per probe CTA)
    long long a = 0;
    for (int r = 0; r < nreg; ++r) { s_pre[r] = a; a += fill[r]; }
    s_pre[nreg] = a;
  }
  __syncthreads();
  const long long total = s_pre[nreg];
  auto fetch = [&](long long v) {                // entry v of the flattened regions (or a hole)
    DEntry d{0, 0, kHole, 0u};
    if (v < total) {
      int lo = 0, hi = nreg;                     // region r: s_pre[r] <= v < s_pre[r + 1]
      while (hi - lo > 1) { const int mid = (lo + hi) >> 1; if (s_pre[mid] <= v) lo = mid; else hi = mid; }
      d = defer[(size_t)lo * cap + (size_t)(v - s_pre[lo])];
    }
    return d;
  };
  const long long gstride = (long long)gridDim.x * 256;
  // software pipeline: the entry two points ahead and the record of the next point are in flight
  // while the current point is tested
  // (pxy != nullptr: the entries hold no coordinates; the point is re-read by its index)
  auto rec_of = [&](DEntry& d, uint32_t& id) {
    if (d.rec == kHole) return Rec{0u, kEmpty, 0, 0u};
    if (pxy) { const int2 q = __ldg(pxy + d.pidx); d.x = q.x; d.y = q.y; }
    if (PIX) d.rec = rec_of_point(cvg, d.x, d.y);   // fine16 canvas: the record from the int32 level
    return load_rec(cvg, d.rec, KAGG ? &id : nullptr);
  };
  DEntry nxt = fetch((long long)blockIdx.x * 256 + threadIdx.x);
  DEntry nxt2 = fetch((long long)blockIdx.x * 256 + gstride + threadIdx.x);
  uint32_t nid = 0;
  Rec nrec = rec_of(nxt, nid);
  for (long long b0 = (long long)blockIdx.x * 256; b0 < total; b0 += gstride) {
    const DEntry e = nxt;
    const Rec rc = nrec;
    const uint32_t rid = nid;
    nxt = nxt2;
    nxt2 = fetch(b0 + 2 * gstride + threadIdx.x);
    nrec = rec_of(nxt, nid);
    const bool act = e.rec != kHole;
    const int64_t pid = o.id_base + (int64_t)e.pidx;
    if ((MODE == kCountSmem || MODE == kCountGlobal) && KAGG) {
      if (act) pip_count_delta<KIND, 4>(cvg, e.x, e.y, rid, rc, kcnt, [&](int q, int d) {
        if (sh) atomicAdd(&dh[q], (unsigned int)d);
        else atomicAdd(o.counts + q, (unsigned long long)(long long)d);
      });
    } else if (MODE == kCountSmem || MODE == kCountGlobal) {
      if (sh) {
        if (act) pip_eval_rec<KIND, 4>(cvg, e.x, e.y, rc, [&](int q) { atomicAdd(&dh[q], 1u); });
      } else {
        // global counts: each point's first result aggregated over the warp (see k_probe)
        int first = -1;
        if (act) pip_eval_rec<KIND, 4>(cvg, e.x, e.y, rc, [&](int q) {
          if (first < 0) first = q; else atomicAdd(o.counts + q, 1ull);
        });
        const unsigned m = __match_any_sync(0xffffffffu, first);
        if (first >= 0 && (m & ((1u << (threadIdx.x & 31)) - 1u)) == 0u)
          atomicAdd(o.counts + first, (unsigned long long)__popc(m));
      }
    } else {
      int nres = 0, first = -1;
      if (act) {
        if (MODE == kSelect) { bool any = false; pip_eval_rec<KIND, 4>(cvg, e.x, e.y, rc, [&](int) { any = true; }); nres = any; }
        else pip_eval_rec<KIND, 4>(cvg, e.x, e.y, rc, [&](int q) { if (nres++ == 0) first = q; });
      }
      int excl, tot;
      BS(tmp).ExclusiveSum(nres, excl, tot);
      if (threadIdx.x == 0) s_gb = tot ? atomicAdd(o.total, (unsigned long long)tot) : 0ull;
      __syncthreads();
      int64_t pos = (int64_t)s_gb + excl;
      if (nres) {
        if (MODE == kSelect) {
          put_result<MODE>(o, pos, pid, 0);
        } else if (nres == 1) {                    // the common case: no second evaluation
          put_result<MODE>(o, pos, pid, first);
        } else {
          pip_eval_rec<KIND>(cvg, e.x, e.y, rc, [&](int q) { put_result<MODE>(o, pos++, pid, q); });
        }
      }
      __syncthreads();
    }
  }
  if (sh) {
    __syncthreads();
    for (int q = threadIdx.x; q < P; q += 256)
      if (dh[q]) atomicAdd(o.counts + q, (unsigned long long)(long long)(int)dh[q]);
  }
}

// Output compaction after a SELECT/PAIRS launch (probe + deferred kernel).  The slots handed out
// are [T0, T); the holes (each warp's unused chunk tail) total H, so the results are M = T - H
// and must end up in [T0, M).  k_fixup (one block) sorts the holes, sets *total = M and lists
// (a) the hole slots below M (destinations, in order) and (b) the runs of result slots at or past
// M (sources, in order); k_move copies the k-th source into the k-th destination.
constexpr int kFixT = 512, kFixItems = 10;
constexpr int kMaxHoles = kFixT * kFixItems;    // warps per launch (grid <= 160 CTAs)
#ifndef SPADE_FIX_RADIX_BITS
#define SPADE_FIX_RADIX_BITS 5
#endif
constexpr int kFixRadixBits = SPADE_FIX_RADIX_BITS;   // digit width of the hole sort's passes
struct FixMeta {
  long long M, nmove;
};

// Sorting the holes by start: relative 32-bit keys with only the bits the range needs (the
// common case), else full 64-bit keys.
template <typename Key>
__device__ __forceinline__ void sort_holes(unsigned long long (&start)[kFixItems], int (&len)[kFixItems],
                                           unsigned long long lo, int bits, void* tmp) {
  using Sort = cub::BlockRadixSort<Key, kFixT, kFixItems, int, kFixRadixBits>;
  Key key[kFixItems];
#pragma unroll
  for (int i = 0; i < kFixItems; ++i) key[i] = (Key)(start[i] - lo);
  Sort(*(typename Sort::TempStorage*)tmp).Sort(key, len, 0, bits);
#pragma unroll
  for (int i = 0; i < kFixItems; ++i) start[i] = lo + (unsigned long long)key[i];
}

__global__ void __launch_bounds__(kFixT) k_fixup(const longlong2* __restrict__ holes, int nh, unsigned long long* total,
                                                 int64_t cap, long long* __restrict__ dst_start,
                                                 long long* __restrict__ dst_pre, long long* __restrict__ src_start,
                                                 long long* __restrict__ src_pre, FixMeta* meta) {
  using Sort32 = cub::BlockRadixSort<unsigned int, kFixT, kFixItems, int, kFixRadixBits>;
  using Sort64 = cub::BlockRadixSort<unsigned long long, kFixT, kFixItems, int, kFixRadixBits>;
  using Scan = cub::BlockScan<long long, kFixT>;
  using Red = cub::BlockReduce<unsigned long long, kFixT>;
  __shared__ union {
    typename Sort32::TempStorage s32;
    typename Sort64::TempStorage s64;
    typename Scan::TempStorage scan;
    typename Red::TempStorage red;
    long long next[kMaxHoles + 1];
  } sm;
  __shared__ unsigned long long s_H, s_lo, s_hi;
  const long long T = (long long)*total;
  unsigned long long st[kFixItems];
  int len[kFixItems];
  unsigned long long hl = 0, lo = ~0ull, hi = 0;
#pragma unroll
  for (int i = 0; i < kFixItems; ++i) {
    const int h = threadIdx.x * kFixItems + i;
    const longlong2 v = h < nh ? holes[h] : make_longlong2(0, 0);
    len[i] = (int)v.y;
    st[i] = v.y > 0 ? (unsigned long long)v.x : ~0ull;       // empty holes: sorted last
    hl += (unsigned long long)v.y;
    if (v.y > 0) { lo = min(lo, (unsigned long long)v.x); hi = max(hi, (unsigned long long)v.x); }
  }
  unsigned long long r = Red(sm.red).Sum(hl);
  if (threadIdx.x == 0) s_H = r;
  __syncthreads();
  r = Red(sm.red).Reduce(lo, cub::Min());
  if (threadIdx.x == 0) s_lo = r;
  __syncthreads();
  r = Red(sm.red).Reduce(hi, cub::Max());
  if (threadIdx.x == 0) s_hi = r;
  __syncthreads();
  const unsigned long long L = s_lo == ~0ull ? 0ull : s_lo, span = s_lo == ~0ull ? 0ull : s_hi - s_lo + 1;
#pragma unroll
  for (int i = 0; i < kFixItems; ++i) if (st[i] == ~0ull) st[i] = L + span;   // empty: past every start
  const int bits = span == 0 ? 1 : 64 - __clzll(span);
  if (bits <= 32) sort_holes<unsigned int>(st, len, L, bits, &sm);
  else sort_holes<unsigned long long>(st, len, L, bits, &sm);
  __syncthreads();
  const long long M = T - (long long)s_H;
  // Hole i = [a, e).  Destinations: its part below M.  Sources: the run of result slots after
  // its part at or past M, [max(e, M), max(a', M)) with a' the next hole's start (T after the
  // last), plus the leading run [M, max(a_0, M)).
#pragma unroll
  for (int i = 0; i < kFixItems; ++i)
    sm.next[threadIdx.x * kFixItems + i] = len[i] > 0 ? max((long long)st[i], M) : T;
  if (threadIdx.x == 0) sm.next[kMaxHoles] = T;
  __syncthreads();
  long long dl[kFixItems], gs[kFixItems], gl[kFixItems];
  long long dsum = 0, gsum = 0;
#pragma unroll
  for (int i = 0; i < kFixItems; ++i) {
    const bool valid = len[i] > 0;
    const long long a = (long long)st[i], e = a + len[i];
    dl[i] = valid && a < M ? min(e, M) - a : 0;
    gs[i] = valid ? max(e, M) : T;
    gl[i] = valid ? max(sm.next[threadIdx.x * kFixItems + i + 1] - gs[i], 0ll) : 0;
    dsum += dl[i];
    gsum += gl[i];
  }
  const long long lead = sm.next[0] - M;
  __syncthreads();                                // sm.next is reused by the scans
  long long dex, gex;
  Scan(sm.scan).ExclusiveSum(dsum, dex);
  __syncthreads();
  Scan(sm.scan).ExclusiveSum(gsum, gex);
#pragma unroll
  for (int i = 0; i < kFixItems; ++i) {
    const int h = threadIdx.x * kFixItems + i;
    dst_start[h] = len[i] > 0 ? (long long)st[i] : T;
    dst_pre[h] = dex;                             // exclusive prefix of destination slots
    dex += dl[i];
    src_start[h + 1] = gs[i];
    src_pre[h + 1] = lead + gex;                  // exclusive prefix of source slots
    gex += gl[i];
  }
  if (threadIdx.x == 0) {
    src_start[0] = M;
    src_pre[0] = 0;
  }
  if (threadIdx.x == kFixT - 1) {
    FixMeta m;
    m.M = M;
    m.nmove = M <= cap ? dex : 0;                 // results lost to capacity: nothing to repair
    *meta = m;
    *total = (unsigned long long)M;
  }
}

// k-th destination slot / source slot: upper-bound searches in the prefix arrays
__device__ __forceinline__ int find_run(const long long* __restrict__ pre, int n, long long k) {
  int lo = 0, hi = n;                            // last i with pre[i] <= k
  while (hi - lo > 1) { const int mid = (lo + hi) >> 1; if (pre[mid] <= k) lo = mid; else hi = mid; }
  return lo;
}

// (the two prefix arrays are copied to shared memory first: the per-slot searches would otherwise
// be ~26 dependent L2 round trips, the whole kernel's duration for small outputs)
template <int MODE>
__global__ void __launch_bounds__(1024) k_move(Out o, const long long* __restrict__ dst_start, const long long* __restrict__ dst_pre_g,
                                               const long long* __restrict__ src_start, const long long* __restrict__ src_pre_g,
                                               const FixMeta* __restrict__ meta) {
  extern __shared__ long long pre_s[];
  long long* dst_pre = pre_s;
  long long* src_pre = pre_s + kMaxHoles;
  const FixMeta m = *meta;
  if (m.nmove == 0) return;
  for (int i = threadIdx.x; i < kMaxHoles; i += blockDim.x) dst_pre[i] = dst_pre_g[i];
  for (int i = threadIdx.x; i < kMaxHoles + 1; i += blockDim.x) src_pre[i] = src_pre_g[i];
  __syncthreads();
  for (long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x; k < m.nmove;
       k += (long long)gridDim.x * blockDim.x) {
    const int di = find_run(dst_pre, kMaxHoles, k);
    const long long d = dst_start[di] + (k - dst_pre[di]);
    const int si = find_run(src_pre, kMaxHoles + 1, k);
    const long long q = src_start[si] + (k - src_pre[si]);
    const bool ov = q >= o.cap;
    const int64_t id = ov ? o.ovf_ids[q - o.cap] : o.out_ids[q];
    o.out_ids[d] = id;                           // d < M <= cap
    if (MODE == kPairs) o.out_poly[d] = ov ? o.ovf_poly[q - o.cap] : o.out_poly[q];
  }
}

// Stream-ordered scratch comes from the device's default memory pool; by default the pool hands
// memory back to the driver at every synchronisation, which made each call re-map its scratch.
// Set once per device (the caller's current device, which the entry points switch to the canvas's).
}  // namespace

void keep_pool_memory() {
  static std::atomic<uint64_t> done{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = 1ull << (dev & 63);
  if (done.fetch_or(bit) & bit) return;
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
    uint64_t thr = 16ull << 30;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  cudaGetLastError();
}

namespace {

// Spread the per-record counts of multi-owner pixels over their owner sets (see count_multi_owner).
// hist != 0: per-block shared-memory bins of all P polygons (P <= 12K), flushed with one global
// atomic per nonzero bin (an owner-set entry is one shared-memory atomic, not one global one).
__global__ void __launch_bounds__(256) k_multi_expand(const CanvasDev* __restrict__ cvg, const unsigned int* __restrict__ rec_cnt,
                                                     uint32_t multi_base, uint32_t num_multi, unsigned long long* counts,
                                                     int hist) {
  extern __shared__ unsigned long long eh[];
  const int P = cvg->num_polys;
  if (hist) {
    for (int i = threadIdx.x; i < P; i += 256) eh[i] = 0ull;
    __syncthreads();
  }
  for (uint32_t i = blockIdx.x * 256 + threadIdx.x; i < num_multi; i += gridDim.x * 256) {
    const unsigned int k = rec_cnt[i];
    if (k == 0u) continue;
    const int32_t term = cvg->recs[multi_base + i].term;
    if (term >= 0) {
      if (hist) atomicAdd(&eh[term], (unsigned long long)k); else atomicAdd(counts + term, (unsigned long long)k);
    } else if (term != kEmpty) {
      const int2 g = cvg->set_rng[-2 - term];
      for (int j = 0; j < g.y; ++j) {
        const int q = cvg->sets[g.x + j];
        if (hist) atomicAdd(&eh[q], (unsigned long long)k); else atomicAdd(counts + q, (unsigned long long)k);
      }
    }
  }
  if (hist) {
    __syncthreads();
    for (int i = threadIdx.x; i < P; i += 256)
      if (eh[i]) atomicAdd(counts + i, eh[i]);
  }
}

// Optional per-stage CUDA events of the last probe call (spade_set_option "stage_events"; read
// with spade_last_call_stages): probe kernel, deferred exact tests, output compaction, per-record
// counter expansion, summed over the call's sub-launches.
struct StageEvents {
  static constexpr int kN = kProbeStages;
  cudaEvent_t ev[kN + 1] = {};
  float acc[kN] = {};
  bool on = false;
  cudaStream_t st = nullptr;
  void begin(cudaStream_t s) {
    on = options().stage_events != 0;
    if (!on) return;
    st = s;
    for (int i = 0; i <= kN; ++i) if (!ev[i]) cudaEventCreate(&ev[i]);
  }
  void rec(int i) { if (on) cudaEventRecord(ev[i], st); }
  void add() {                                    // after rec(0..kN) of one sub-launch: accumulate
    if (!on) return;
    cudaEventSynchronize(ev[kN]);
    for (int i = 0; i < kN; ++i) { float ms = 0.f; cudaEventElapsedTime(&ms, ev[i], ev[i + 1]); acc[i] += ms; }
  }
};
thread_local StageEvents g_stages;

// Stream-ordered device scratch freed on every exit path (errors included).
struct ScratchGuard {
  void* p = nullptr;
  cudaStream_t st = nullptr;
  ~ScratchGuard() { if (p) cudaFreeAsync(p, st); }
};

// COUNT with K aggregation (boundary points counted per record for the corner set K): heavily
// overlapping polygon sets
bool kagg_for(const spade_canvas* c) {
  const int o = options().k_agg;
  return c->num_runs > 0 && (o == 1 || (o < 0 && 2 * c->num_set_entries > c->num_records));
}

template <int MODE, int COMPACT, int QUEUE, int KIND, int PIPE = 0>
int launch(const spade_canvas* c, const int2* xy, int64_t n, const Params& base, size_t extra_smem, cudaStream_t st) {
  const size_t base_smem = PIPE == 2 ? ((extra_smem + 15) & ~(size_t)15) + pipe_ring_bytes(kPipeNoTileD)
                         : PIPE ? tiles_bytes_for(c->d.Wc, c->d.Hc) + ((extra_smem + 15) & ~(size_t)15) + pipe_ring_bytes()
                                : tiles_bytes_for(c->d.Wc, c->d.Hc) + extra_smem + (QUEUE ? queue_bytes(MODE, QUEUE) : 0);
  // TMA stages (1 KB per warp + mbarriers) after everything else, 128-B aligned; the smem_pad_kb
  // option adds the same amount of unused shared memory to other variants (equal-footprint A/B)
  const size_t tma_off = (base_smem + 127) & ~(size_t)127;
  const size_t smem = QUEUE == 2 ? tma_off + (size_t)kNW * (1024 + 8) : base_smem + (size_t)options().smem_pad_kb * 1024;
  void (*kern)(const Params);
  if constexpr (PIPE == 2) kern = k_probe_pipe<MODE, COMPACT, KIND, 2>;
  else if constexpr (PIPE != 0) kern = k_probe_pipe<MODE, COMPACT, KIND, 1>;
  else kern = k_probe<MODE, COMPACT, QUEUE, KIND>;
  // (the attribute is set when it grows, once per device and instantiation: a driver call per
  // probe call showed as host latency on short calls)
  static std::atomic<int> smem_set[16];
  int dev = 0;
  cudaGetDevice(&dev);
  cudaError_t e = cudaSuccess;
  if (smem_set[dev & 15].load(std::memory_order_relaxed) < (int)smem) {
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return check_cuda(e, "probe smem attribute");
    int cur = smem_set[dev & 15].load();
    while (cur < (int)smem && !smem_set[dev & 15].compare_exchange_weak(cur, (int)smem)) {}
  }
  const int sms = device_sm_count();
  keep_pool_memory();
  g_stages.begin(st);
  // COUNT over a canvas with multi-owner pixels: per-record counters (count_multi_owner)
  constexpr bool kCnt = MODE == kCountSmem || MODE == kCountGlobal;
  const uint32_t num_multi = kCnt && options().multi_agg ? (uint32_t)(c->num_records - c->num_runs) : 0u;
  ScratchGuard rec_g, kcnt_g;
  rec_g.st = kcnt_g.st = st;
  unsigned int* rec_cnt = nullptr;
  if (num_multi > 0) {
    e = cudaMallocAsync((void**)&rec_cnt, sizeof(unsigned int) * num_multi, st);
    if (e != cudaSuccess) return check_cuda(e, "multi-owner counters");
    rec_g.p = rec_cnt;
    e = cudaMemsetAsync(rec_cnt, 0, sizeof(unsigned int) * num_multi, st);
    if (e != cudaSuccess) return check_cuda(e, "multi-owner counters");
  }
  // COUNT over heavily overlapping polygons (owner sets much larger than one polygon on average):
  // boundary points counted per record for the term set K + per-point parity deltas
  const bool kagg = kCnt && kagg_for(c);
  unsigned int* kcnt = nullptr;
  if (options().debug_defer)
    fprintf(stderr, "[spade] records %lld (boundary %lld), set entries %lld, k_agg %d\n", (long long)c->num_records,
            (long long)c->num_runs, (long long)c->num_set_entries, (int)kagg);
  if (kagg) {
    // every record: multi-owner records reach the exact-test paths too when multi_agg is off
    e = cudaMallocAsync((void**)&kcnt, sizeof(unsigned int) * c->num_records, st);
    if (e != cudaSuccess) return check_cuda(e, "boundary-record counters");
    kcnt_g.p = kcnt;
    e = cudaMemsetAsync(kcnt, 0, sizeof(unsigned int) * c->num_records, st);
    if (e != cudaSuccess) return check_cuda(e, "boundary-record counters");
  }
  // The per-record counters are uint32: they are spread over the owner sets (and cleared) after
  // every sub-launch, each of which holds < 2^31 points, so no counter can wrap whatever n is.
  if (kcnt || rec_cnt) cudaFuncSetAttribute(k_multi_expand, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * 12288);
  auto expand = [&](bool clear) -> int {
    if (kcnt) {
      const int g = (int)std::min<int64_t>((int64_t)sms * 8, (c->num_records + 255) / 256);
      const int eh = c->d.num_polys <= 12288;
      k_multi_expand<<<g, 256, eh ? 8 * c->d.num_polys : 0, st>>>(c->d_dev, kcnt, 0u, (uint32_t)c->num_records, base.o.counts, eh);
      count_launch();
      cudaError_t e2 = cudaGetLastError();
      if (e2 == cudaSuccess && clear) e2 = cudaMemsetAsync(kcnt, 0, sizeof(unsigned int) * c->num_records, st);
      if (e2 != cudaSuccess) return check_cuda(e2, "boundary-record expand");
    }
    if (rec_cnt) {
      const int g = (int)std::min<int64_t>((int64_t)sms * 8, ((int64_t)num_multi + 255) / 256);
      const int eh = c->d.num_polys <= 12288;
      k_multi_expand<<<g, 256, eh ? 8 * c->d.num_polys : 0, st>>>(c->d_dev, rec_cnt, (uint32_t)c->num_runs, num_multi, base.o.counts, eh);
      count_launch();
      cudaError_t e2 = cudaGetLastError();
      if (e2 == cudaSuccess && clear) e2 = cudaMemsetAsync(rec_cnt, 0, sizeof(unsigned int) * num_multi, st);
      if (e2 != cudaSuccess) return check_cuda(e2, "multi-owner expand");
    }
    return SPADE_OK;
  };
  // Sub-launches of fewer than 2^31 points (32-bit vector indices, point offsets and per-record
  // counters).  Deferral regions are sized from the canvas's boundary-pixel fraction fb (points
  // are not uniform, so 2 fb + 4%, at most all points; overflowing points are tested in place),
  // 16 B per entry; a sub-launch is also cut so that its regions stay within the deferral budget
  // (spade_set_option "defer_budget_mb"), which bounds the scratch for boundary-heavy canvases.
  const double fb = (double)c->num_runs / ((double)c->d.W * (double)c->d.H);
  const double frac = std::min(1.0, 2.0 * fb + 0.04);
  int64_t kMax = std::min<int64_t>((1ll << 31) - 64, options().max_launch_points);
  if (!QUEUE) {
    const double budget = (double)options().defer_budget_mb * (1 << 20);
    kMax = std::min<int64_t>(kMax, std::max<int64_t>(1 << 16, (int64_t)(budget / (16.0 * frac))));
  }
  for (int64_t off = 0; off < n; off += kMax) {
    const int64_t m = std::min(kMax, n - off);
    Params p = base;
    p.xy = xy + off;
    p.n = m;
    const uintptr_t addr = (uintptr_t)p.xy;
    p.head = std::min<int64_t>(m, (int64_t)(((32 - (addr & 31)) & 31) / 8));
    p.nvec = (m - p.head) / 4;
    p.o.id_base = base.o.id_base + off;
    const int64_t chunks = (p.nvec + kT - 1) / kT;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(std::min(sms, kMaxHoles / kNW), chunks));
    const int64_t per = QUEUE ? 0 : std::min<int64_t>(std::max<int64_t>((int64_t)(frac * (double)m / grid) + 64, 1024),
                                                       (int64_t)1 << 26);
    // SELECT/PAIRS: warp output chunks of K slots (about 1/16 of a warp's points, 256..2048),
    // overflow slots for every warp's possible hole, hole list and compaction tables
    constexpr bool kOut = MODE == kSelect || MODE == kPairs;
    uint32_t K = 0;
    if (kOut) {
      const int64_t per_warp = m / ((int64_t)grid * kNW) / 16;
      K = 256;
      while (K < 2048 && (int64_t)K * 2 <= per_warp) K *= 2;
    }
    const int64_t ovf = kOut ? (int64_t)grid * kNW * K : 0;
    size_t sz[9] = {sizeof(DEntry) * (QUEUE ? 0 : per * grid), QUEUE ? 0 : sizeof(unsigned int) * grid,
                    sizeof(int64_t) * ovf, MODE == kPairs ? sizeof(int32_t) * ovf : 0,
                    kOut ? sizeof(longlong2) * kMaxHoles : 0, kOut ? 8 * (size_t)kMaxHoles : 0,
                    kOut ? 8 * (size_t)kMaxHoles : 0, kOut ? 8 * (size_t)(kMaxHoles + 1) : 0,
                    kOut ? 8 * (size_t)(kMaxHoles + 1) + sizeof(FixMeta) : 0};
    size_t total_sz = 0, offs[9];
    for (int i = 0; i < 9; ++i) { offs[i] = total_sz; total_sz += (sz[i] + 255) & ~(size_t)255; }
    ScratchGuard scr;
    scr.st = st;
    unsigned char* scratch = nullptr;
    if (total_sz > 0) {
      e = cudaMallocAsync((void**)&scratch, total_sz, st);
      if (e != cudaSuccess) return check_cuda(e, "probe scratch");
      scr.p = scratch;
    }
    DEntry* dbuf = QUEUE ? nullptr : (DEntry*)(scratch + offs[0]);
    unsigned int* dfill = QUEUE ? nullptr : (unsigned int*)(scratch + offs[1]);
    long long* fix_ds = (long long*)(scratch + offs[5]);
    long long* fix_dp = (long long*)(scratch + offs[6]);
    long long* fix_ss = (long long*)(scratch + offs[7]);
    long long* fix_sp = (long long*)(scratch + offs[8]);
    FixMeta* fix_meta = (FixMeta*)(scratch + offs[8] + 8 * (size_t)(kMaxHoles + 1));
    if (kOut) {
      p.o.chunk = K;
      p.o.ovf_ids = (int64_t*)(scratch + offs[2]);
      p.o.ovf_poly = MODE == kPairs ? (int32_t*)(scratch + offs[3]) : nullptr;
      p.o.ovf_cap = ovf;
      p.o.holes = (longlong2*)(scratch + offs[4]);
    }
    p.defer = dbuf;
    p.defer_xy = PIPE ? (uint32_t)options().defer_xy : 0u;
    p.rec_cnt = rec_cnt;
    p.multi_base = (uint32_t)c->multi_unit;
    p.kcnt = kcnt;
    p.l2_frac = (float)options().l2_frac_pct * 0.01f;
    p.defer_cap = (uint32_t)per;
    p.defer_fill = dfill;
    p.tma_off = (uint32_t)tma_off;
    g_stages.rec(0);
    kern<<<grid, kT, smem, st>>>(p);
    count_launch();
    e = cudaGetLastError();
    g_stages.rec(1);
    if (e == cudaSuccess && !QUEUE) {
      const int P = c->d.num_polys;
      const int sh = ((MODE == kCountSmem || MODE == kCountGlobal) && (size_t)P * 4 <= 96 * 1024) ? 1 : 0;
      const size_t dsm = sh ? (size_t)P * 4 : 0;
      const int coop = options().coop;
      bool launched = false;
      if constexpr (MODE == kCountSmem || MODE == kCountGlobal) if (coop != 0) {
        // cooperative groups sized to the records' mean primitive count (4 / 8 / 16 lanes)
        const double epr = c->num_runs ? (double)c->num_run_edges / (double)c->num_runs : 1.0;
        const int G = coop > 0 ? coop : (epr > 10.0 ? 16 : epr > 4.0 ? 8 : 4);
        const int hs = (size_t)P * 4 <= 200 * 1024 ? 1 : 0;
        const size_t hsm = hs ? (size_t)P * 4 : 0;
        constexpr int PX = COMPACT == 2;
        auto kd = G >= 16 ? k_deferred_count<MODE, KIND, 16, PX> : G >= 8 ? k_deferred_count<MODE, KIND, 8, PX> : k_deferred_count<MODE, KIND, 4, PX>;
        cudaFuncSetAttribute(kd, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)std::max<size_t>(hsm, 1));
        kd<<<sms, 1024, hsm, st>>>(c->d_dev, dbuf, p.defer_cap, dfill, grid, p.o.counts, hs,
                                   PIPE && !p.defer_xy ? p.xy : nullptr);
        launched = true;
      }
      if (!launched) {
        constexpr int PX = COMPACT == 2;
        auto kd = kcnt ? k_deferred<MODE, KIND, PX, (MODE == kCountSmem || MODE == kCountGlobal)> : k_deferred<MODE, KIND, PX, 0>;
        if (dsm > 48 * 1024) cudaFuncSetAttribute(kd, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsm);
        kd<<<sms * 8, 256, dsm, st>>>(c->d_dev, dbuf, p.defer_cap, dfill, grid, p.o, sh,
                                      PIPE && !p.defer_xy ? p.xy : nullptr, kcnt);
      }
      count_launch();
      e = cudaGetLastError();
      const bool dbg = options().debug_defer != 0;
      if (dbg && e == cudaSuccess) {           // diagnostics only: synchronises
        std::vector<unsigned int> f(grid);
        cudaMemcpyAsync(f.data(), dfill, sizeof(unsigned int) * grid, cudaMemcpyDeviceToHost, st);
        cudaStreamSynchronize(st);
        long long tot = 0; unsigned int mx = 0;
        for (unsigned int x : f) { tot += x; mx = std::max(mx, x); }
        fprintf(stderr, "[spade] deferred %lld of %lld points (%.2f%%), max region %u of cap %lld, runs %lld, run edges %lld\n",
                tot, (long long)m, 100.0 * tot / m, mx, (long long)per, (long long)c->num_runs, (long long)c->num_run_edges);
      }
    }
    g_stages.rec(2);
    if (kOut && e == cudaSuccess) {
      k_fixup<<<1, kFixT, 0, st>>>(p.o.holes, grid * kNW, p.o.total, p.o.cap, fix_ds, fix_dp, fix_ss, fix_sp, fix_meta);
      count_launch();
      const int msm = (int)(sizeof(long long) * (2 * kMaxHoles + 1));
      static std::atomic<uint32_t> move_set{0};          // (bit per device: set once)
      if (!(move_set.load(std::memory_order_relaxed) & (1u << (dev & 15)))) {
        cudaFuncSetAttribute(k_move<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, msm);
        move_set.fetch_or(1u << (dev & 15));
      }
      k_move<MODE><<<sms, 1024, msm, st>>>(p.o, fix_ds, fix_dp, fix_ss, fix_sp, fix_meta);
      count_launch();
      e = cudaGetLastError();
    }
    g_stages.rec(3);
    if (e != cudaSuccess) return check_cuda(e, "probe launch");
    const int rc = expand(off + m < n);
    if (rc != SPADE_OK) return rc;
    g_stages.rec(4);
    g_stages.add();
  }
  return SPADE_OK;
}

template <int MODE, int QUEUE = 0, int PIPE = 0>
int launch_layout(const spade_canvas* c, const int2* xy, int64_t n, const Params& p, size_t extra, cudaStream_t st) {
  // second level: 2 = dense uint16 (fine16), 1 = compact int32, 0 = dense int32
  const bool f16 = c->d.f16 && options().fine16;
  if (c->d.kind == kDisks) {
    if (f16) return launch<MODE, 2, QUEUE, kDisks, PIPE>(c, xy, n, p, extra, st);
    return c->d.compact ? launch<MODE, 1, QUEUE, kDisks, PIPE>(c, xy, n, p, extra, st) : launch<MODE, 0, QUEUE, kDisks, PIPE>(c, xy, n, p, extra, st);
  }
  if (f16) return launch<MODE, 2, QUEUE, kPolygons, PIPE>(c, xy, n, p, extra, st);
  return c->d.compact ? launch<MODE, 1, QUEUE, kPolygons, PIPE>(c, xy, n, p, extra, st)
                      : launch<MODE, 0, QUEUE, kPolygons, PIPE>(c, xy, n, p, extra, st);
}

Params base_params(const spade_canvas* c) {
  Params p{};
  p.cv = c->d;
  p.cvg = c->d_dev;
  p.hcopies = 1;
  // (wraps below cfine: only ever offset back into it by a tile entry's 0x8000 << 2b)
  if (c->d.compact) p.cfine_tile0 = (const int32_t*)((uintptr_t)c->d.cfine - ((uintptr_t)kTileMixedCompact << (2 * c->d.b)) * 4u);
  return p;
}

// SELECT/PAIRS: boundary points tested in the loop (warp queues) when the queues fit beside the
// tiles; SPADE_DEFER=1 forces the deferral kernel (A/B switch)
bool use_queue(const spade_canvas* c, int mode) {
  return !options().defer && tiles_bytes_for(c->d.Wc, c->d.Hc) + queue_bytes(mode) <= kSmemSoft;
}

}  // namespace

int last_call_stages(float* ms, int cap) {
  int n = 0;
  for (; n < kProbeStages && n < cap; ++n) ms[n] = g_stages.acc[n];
  return kProbeStages;
}
void reset_call_stages() { for (float& a : g_stages.acc) a = 0.f; }

int launch_count(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t* counts, cudaStream_t st) {
  reset_call_stages();
  if (c->empty || n == 0) return SPADE_OK;
  Params p = base_params(c);
  p.o.counts = (unsigned long long*)counts;
  // shared-memory histogram: as many copies (8, 4, 2, 1) as stay under the L1-preserving budget;
  // boundary points tested in the loop (warp queues) when those fit too, else deferred
  const size_t tiles = tiles_bytes_for(c->d.Wc, c->d.Hc);
  const size_t one = (size_t)(c->d.num_polys + 1) * 4;
  // shared memory of hc histogram copies, rounded up to 16 B (what follows is 8- or 16-B aligned)
  auto hb = [&](uint32_t hc) { return ((size_t)hc * one + 15) & ~(size_t)15; };
  const size_t queue = queue_bytes(kCountSmem);
  const int force_defer = options().defer, force_global = options().count_global;
  // Mostly-mixed canvases whose only shared-memory histogram option is a single copy filling
  // the budget (C5: 40k polygons) take the cp.async-pipelined probe with global counters, which
  // keeps the L1 carve-out (measured: C5 14.2 -> 13.6 ms; dj2, global counters either way, is
  // slower with it: 23.1 -> 25.7 ms)
  const int pipe_opt = options().pipe;
  const bool pipe_auto = c->mixed_tile_frac > 0.5 && tiles + 2 * one > kSmemSoft && tiles + one <= 227 * 1024;
  if (pipe_opt == 1 || (pipe_opt < 0 && pipe_auto && !force_defer && !force_global)) {
    // every tile mixed and a dense second level: the tile-less variant with a full histogram
    if (options().pipe_notile && c->mixed_tile_frac >= 0.999 && !c->d.compact && !force_global) {
      const size_t ring2 = pipe_ring_bytes(kPipeNoTileD);
      for (uint32_t hc = 8; hc >= 1; hc >>= 1)
        if (((hb(hc) + 15) & ~(size_t)15) + ring2 <= kPipeSmem) {
          p.hcopies = hc;
          return launch_layout<kCountSmem, 0, 2>(c, (const int2*)xy, n, p, hb(hc), st);
        }
    }
    const size_t ring = pipe_ring_bytes();
    for (uint32_t hc = 8; hc >= 1 && !force_global; hc >>= 1) {
      if (tiles + ((hb(hc) + 15) & ~(size_t)15) + ring <= kPipeSmem) {
        p.hcopies = hc;
        return launch_layout<kCountSmem, 0, 1>(c, (const int2*)xy, n, p, hb(hc), st);
      }
    }
    uint32_t slots = 0;
    for (uint32_t ns = (uint32_t)options().cache_slots; ns >= 1024; ns >>= 1)
      if (tiles + (size_t)ns * 8 + ring <= kSmemSoft) { slots = ns; break; }
    if (tiles + (size_t)slots * 8 + ring <= 227 * 1024) {
      p.cache_slots = slots;
      return launch_layout<kCountGlobal, 0, 1>(c, (const int2*)xy, n, p, (size_t)slots * 8, st);
    }
  }
  // Histogram copies: copy = lane & (hc - 1) at bin·hc + copy, so with 32 copies every lane of
  // a warp increments its own bank (the histogram atomics were the largest share of C3's
  // shared-memory wavefronts: 124M of 240M, 88M of them bank conflicts, at 8 copies).  A queue of
  // 4-B point indices (the drain re-reads its points) makes room for them beside big tile grids.
  const uint32_t hmax = (uint32_t)options().hist_copies_max;
  const int idxq = options().idx_queue;
  // Overlap-heavy (K-aggregated) canvases: the exact tests walk records for a third of the points,
  // and the L1 that serves those walks grows in steps with the shared memory left free (the
  // carve-out); auto (-1) takes 4-B index queues and as many histogram copies as keep the CTA at
  // or below the 164 KB step (measured: ov 29.2 -> 27.1 ms; C3 and C4, which re-read few queued
  // points but gather more, are faster with point queues and stay on them).
  if (idxq < 0 && !force_defer && !force_global && kagg_for(c))
    for (uint32_t hc = hmax; hc >= 1; hc >>= 1)
      if (tiles + hb(hc) + queue_bytes(kCountSmem, 3) <= kSmemL1Step) {
        p.hcopies = hc;
        return launch_layout<kCountSmem, 3>(c, (const int2*)xy, n, p, hb(hc), st);
      }
  for (uint32_t hc = hmax; hc >= 1 && !force_global; hc >>= 1) {
    if (!force_defer && idxq != 1 && tiles + hb(hc) + queue <= kSmemSoft) {
      p.hcopies = hc;
      // A/B option "tma": the same launch with the point stream staged by TMA (+33 KB of stages)
      if (options().tma) {
        // the TMA variant (index queue + 33 KB of stages) with as many histogram copies as fit
        for (uint32_t ht = hc; ht >= 1; ht >>= 1)
          if (tiles + hb(ht) + queue_bytes(kCountSmem, 2) + 128 + (size_t)kNW * 1032 <= kSmemSoft + options().tma_slack_kb * 1024) {
            p.hcopies = ht;
            return launch_layout<kCountSmem, 2>(c, (const int2*)xy, n, p, hb(ht), st);
          }
      }
      return launch_layout<kCountSmem, 1>(c, (const int2*)xy, n, p, hb(hc), st);
    }
    if (!force_defer && idxq == 1 && tiles + hb(hc) + queue_bytes(kCountSmem, 3) <= kSmemSoft) {
      p.hcopies = hc;
      return launch_layout<kCountSmem, 3>(c, (const int2*)xy, n, p, hb(hc), st);
    }
  }
  for (uint32_t hc = 8; hc >= 1 && !force_global; hc >>= 1) {
    if (tiles + hb(hc) <= kSmemSoft || (hc == 1 && tiles + one <= 227 * 1024)) {
      p.hcopies = hc;
      return launch_layout<kCountSmem>(c, (const int2*)xy, n, p, hb(hc), st);
    }
  }
  // global counts with a shared-memory count cache in the space the tiles leave
  // (boundary points tested in the loop when the warp queues fit too)
  const int max_slots = options().cache_slots;
  // (measured on C5 / dj2: in-loop tests 3-12% slower than deferral; opt in with SPADE_GLOBAL_QUEUE=1)
  const int global_queue = options().global_queue;
  const size_t gq = (force_defer || !global_queue) ? SIZE_MAX / 2 : queue;
  uint32_t slots = 0;
  for (uint32_t ns = (uint32_t)max_slots; ns >= 1024; ns >>= 1)
    if (tiles + gq + (size_t)ns * 8 <= kSmemSoft) { slots = ns; break; }
  if (slots || tiles + gq <= kSmemSoft) {
    p.cache_slots = slots;
    return launch_layout<kCountGlobal, 1>(c, (const int2*)xy, n, p, (size_t)slots * 8, st);
  }
  for (uint32_t ns = (uint32_t)max_slots; ns >= 1024; ns >>= 1)
    if (tiles + (size_t)ns * 8 <= kSmemSoft) { slots = ns; break; }
  p.cache_slots = slots;
  return launch_layout<kCountGlobal>(c, (const int2*)xy, n, p, (size_t)slots * 8, st);
}

int launch_select(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t base, int64_t* out, int64_t cap,
                  unsigned long long* d_total, cudaStream_t st) {
  reset_call_stages();
  if (c->empty || n == 0) return SPADE_OK;
  Params p = base_params(c);
  p.o.id_base = base; p.o.out_ids = out; p.o.cap = cap; p.o.total = d_total;
  if (use_queue(c, kSelect)) return launch_layout<kSelect, 1>(c, (const int2*)xy, n, p, 0, st);
  return launch_layout<kSelect>(c, (const int2*)xy, n, p, 0, st);
}

int launch_pairs(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t base, int64_t* opt, int32_t* opl,
                 int64_t cap, unsigned long long* d_total, cudaStream_t st) {
  reset_call_stages();
  if (c->empty || n == 0) return SPADE_OK;
  Params p = base_params(c);
  p.o.id_base = base; p.o.out_ids = opt; p.o.out_poly = opl; p.o.cap = cap; p.o.total = d_total;
  if (use_queue(c, kPairs)) return launch_layout<kPairs, 1>(c, (const int2*)xy, n, p, 0, st);
  return launch_layout<kPairs>(c, (const int2*)xy, n, p, 0, st);
}

}  // namespace spade
