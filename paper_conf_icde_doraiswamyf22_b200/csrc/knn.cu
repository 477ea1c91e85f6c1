// knn.cu — kNN selection over points (Sec. 5.2 "kNN Queries"), B200 design.
//
// The paper's 3-step plan for the k points nearest to a query point q:
//   1. aggregation (COUNT) of the data over a set of concentric circles around q with radii
//      r_i = r_max / alpha^i  ("one pass over the constraints irrespective of their number");
//   2. a distance selection with the smallest circle whose count is >= k;
//   3. sort the selected points by distance to q and keep the first k.
// Here the circle set is chosen so that step 1 is a pure bit operation per point: the squared
// radii are the upper ends of "quarter-octave" buckets of the squared distance,
//   bucket(d2) = d2                                  for d2 < 4
//              = 4 + 4 (e - 2) + ((d2 >> (e-2)) & 3)  for d2 >= 4,  e = floor(log2 d2)
// so circle b has r2_b = the largest d2 of bucket b (consecutive radii differ by a factor
// alpha <= sqrt(1.25)), and COUNT(circle b) = sum of the bucket histogram up to b.  A canvas of
// nested circles would give every pixel an owner set of up to 248 circles; the bucket histogram
// is the same aggregation with one shared-memory atomic per point.
//
// Step 1 is k_knn_hist (streaming, HBM-bound), step 2 k_knn_select (streaming, HBM-bound, a few
// candidates written), step 3 a radix sort of the candidates by (dist2, point id).
#include <cstdint>
#include <algorithm>
#include <vector>
#include <cub/cub.cuh>
#include "spade_internal.cuh"

namespace spade {

namespace {

constexpr int kKT = 512;              // threads per CTA
constexpr int kHistCopies = 8;

struct alignas(32) P4 { int4 a, b; };   // 4 points

__device__ __forceinline__ P4 ld_stream4(const P4* p) {
  P4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r.a.x), "=r"(r.a.y), "=r"(r.a.z), "=r"(r.a.w), "=r"(r.b.x), "=r"(r.b.y), "=r"(r.b.z),
                 "=r"(r.b.w)
               : "l"(p));
  return r;
}

__host__ __device__ __forceinline__ int knn_bucket(uint64_t d2) {
#ifdef __CUDA_ARCH__
  if (d2 < 4) return (int)d2;
  const int e = 63 - __clzll((long long)d2);
#else
  if (d2 < 4) return (int)d2;
  const int e = 63 - __builtin_clzll(d2);
#endif
  return 4 + 4 * (e - 2) + (int)((d2 >> (e - 2)) & 3u);
}

// a point is in the kNN coordinate range iff both coordinates lie in [-2^30, 2^30)
__device__ __forceinline__ bool in_range(int x, int y) {
  return ((uint32_t)x + (1u << 30) < (1u << 31)) && ((uint32_t)y + (1u << 30) < (1u << 31));
}

// exact squared distance (< 2^63 for in-range coordinates); dx, dy fit in int32
__device__ __forceinline__ uint64_t dist2(int x, int y, int qx, int qy) {
  const int dx = x - qx, dy = y - qy;
  return (uint64_t)((long long)dx * dx) + (uint64_t)((long long)dy * dy);
}

struct Stream {
  const int2* xy;
  int64_t n, head, nvec;     // head: points before the first 32-B aligned one
};

Stream make_stream(const int32_t* xy, int64_t n) {
  Stream s;
  s.xy = (const int2*)xy;
  s.n = n;
  s.head = std::min<int64_t>(n, (int64_t)(((32 - ((uintptr_t)xy & 31)) & 31) / 8));
  s.nvec = (n - s.head) / 4;
  return s;
}

// Step 1: per-bucket counts (hist[kKnnBins]) and out-of-range points (hist[kKnnBins]).
__global__ void __launch_bounds__(kKT) k_knn_hist(Stream s, int qx, int qy, unsigned long long* __restrict__ hist) {
  __shared__ unsigned int h[kHistCopies][kKnnBins + 1];
  for (int i = threadIdx.x; i < kHistCopies * (kKnnBins + 1); i += kKT) (&h[0][0])[i] = 0u;
  __syncthreads();
  unsigned int* mh = h[threadIdx.x & (kHistCopies - 1)];
  auto one = [&](int x, int y) {
    atomicAdd(&mh[in_range(x, y) ? knn_bucket(dist2(x, y, qx, qy)) : kKnnBins], 1u);
  };
  const P4* vp = (const P4*)(s.xy + s.head);
  const int64_t stride = (int64_t)gridDim.x * kKT;
  int64_t i = (int64_t)blockIdx.x * kKT + threadIdx.x;
  P4 nxt;
  if (i < s.nvec) nxt = ld_stream4(vp + i);
  for (; i < s.nvec; i += stride) {
    const P4 v = nxt;
    if (i + stride < s.nvec) nxt = ld_stream4(vp + i + stride);   // next batch in flight
    one(v.a.x, v.a.y); one(v.a.z, v.a.w); one(v.b.x, v.b.y); one(v.b.z, v.b.w);
  }
  if (blockIdx.x == 0 && threadIdx.x < 8) {                        // unaligned head / tail
    const int64_t t0 = s.head + 4 * s.nvec;
    const int64_t j = threadIdx.x < 4 ? threadIdx.x : t0 + (threadIdx.x - 4);
    if ((threadIdx.x < 4 && j < s.head) || (threadIdx.x >= 4 && j < s.n)) { const int2 p = s.xy[j]; one(p.x, p.y); }
  }
  __syncthreads();
  for (int b = threadIdx.x; b <= kKnnBins; b += kKT) {
    unsigned long long t = 0;
    for (int c = 0; c < kHistCopies; ++c) t += h[c][b];
    if (t) atomicAdd(hist + b, t);
  }
}

// Step 2: candidates with dist2 <= r2 (in range), warp-aggregated slot reservation.
__global__ void __launch_bounds__(kKT) k_knn_select(Stream s, int qx, int qy, uint64_t r2, int64_t base,
                                                    int64_t* __restrict__ out_ids, int64_t* __restrict__ out_d2,
                                                    int64_t cap, unsigned long long* __restrict__ total) {
  const int lane = threadIdx.x & 31;
  auto emit = [&](bool hit, int64_t idx, uint64_t d2) {
    const unsigned m = __ballot_sync(0xffffffffu, hit);
    if (!m) return;
    unsigned long long b0 = 0;
    if (lane == 0) b0 = atomicAdd(total, (unsigned long long)__popc(m));
    b0 = __shfl_sync(0xffffffffu, b0, 0);
    if (hit) {
      const int64_t pos = (int64_t)b0 + __popc(m & ((1u << lane) - 1u));
      if (pos < cap) { out_ids[pos] = base + idx; out_d2[pos] = (int64_t)d2; }
    }
  };
  auto test = [&](int x, int y, int64_t idx) {
    const uint64_t d2 = dist2(x, y, qx, qy);
    emit(in_range(x, y) && d2 <= r2, idx, d2);
  };
  const P4* vp = (const P4*)(s.xy + s.head);
  const int64_t stride = (int64_t)gridDim.x * kKT;
  // whole warps iterate together (the emit ballots are warp-wide)
  const int64_t iters = (s.nvec + stride - 1) / stride;
  int64_t i = (int64_t)blockIdx.x * kKT + threadIdx.x;
  P4 nxt;
  if (i < s.nvec) nxt = ld_stream4(vp + i);
  for (int64_t it = 0; it < iters; ++it, i += stride) {
    const bool ok = i < s.nvec;
    P4 v = nxt;
    if (i + stride < s.nvec) nxt = ld_stream4(vp + i + stride);
    if (!ok) { v.a = make_int4(INT32_MIN, INT32_MIN, INT32_MIN, INT32_MIN); v.b = v.a; }   // out of range: no hit
    const int64_t p0 = s.head + 4 * i;
    test(v.a.x, v.a.y, p0); test(v.a.z, v.a.w, p0 + 1); test(v.b.x, v.b.y, p0 + 2); test(v.b.z, v.b.w, p0 + 3);
  }
  if (blockIdx.x == 0 && threadIdx.x < 32) {                       // unaligned head / tail (warp 0)
    const int64_t t0 = s.head + 4 * s.nvec;
    const int64_t j = lane < 4 ? lane : t0 + (lane - 4);
    const bool ok = (lane < 4 && j < s.head) || (lane >= 4 && lane < 8 && j < s.n);
    const int2 p = ok ? s.xy[j] : make_int2(INT32_MIN, INT32_MIN);
    test(p.x, p.y, j);
  }
}

__global__ void k_copy_topk(const int64_t* __restrict__ ids, const int64_t* __restrict__ d2, int64_t k,
                            int64_t* __restrict__ out_ids, int64_t* __restrict__ out_d2) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < k; t += (int64_t)gridDim.x * blockDim.x) {
    out_ids[t] = ids[t];
    if (out_d2) out_d2[t] = d2[t];
  }
}

int grid_stream() { return device_sm_count() * 4; }

}  // namespace

uint64_t knn_bucket_r2(int b) {   // the largest squared distance of bucket b (circle b's r2)
  if (b < 4) return (uint64_t)b;
  const int e = 2 + (b - 4) / 4, j = (b - 4) % 4;
  return (1ull << e) + (uint64_t)(j + 1) * (1ull << (e - 2)) - 1ull;
}

int knn_hist(const int32_t* xy, int64_t n, int32_t qx, int32_t qy, int64_t* hist, cudaStream_t st) {
  if (n == 0) return SPADE_OK;
  const Stream s = make_stream(xy, n);
  k_knn_hist<<<grid_stream(), kKT, 0, st>>>(s, qx, qy, (unsigned long long*)hist);
  count_launch();
  return check_cuda(cudaGetLastError(), "knn histogram");
}

int knn_select(const int32_t* xy, int64_t n, int64_t base, int32_t qx, int32_t qy, uint64_t r2, int64_t* out_ids,
               int64_t* out_d2, int64_t cap, unsigned long long* d_total, cudaStream_t st) {
  if (n == 0) return SPADE_OK;
  const Stream s = make_stream(xy, n);
  k_knn_select<<<grid_stream(), kKT, 0, st>>>(s, qx, qy, r2, base, out_ids, out_d2, cap, d_total);
  count_launch();
  return check_cuda(cudaGetLastError(), "knn select");
}

// Step 3: sort m candidates by (dist2, id) — radix sort by id, then a stable radix sort by
// dist2 — and copy the first min(k, m).
int knn_topk(const int64_t* ids, const int64_t* d2, int64_t m, int64_t k, int64_t* out_ids, int64_t* out_d2,
             cudaStream_t st) {
  if (m == 0 || k == 0) return SPADE_OK;
  if (m >= (1ll << 31)) return set_error(SPADE_ERR_INVALID_ARG, "spade_knn_topk: too many candidates");
  const int mm = (int)m;
  int64_t *k1 = nullptr, *v1 = nullptr, *k2 = nullptr, *v2 = nullptr;
  void* tmp = nullptr;
  size_t ta = 0, tb = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, ta, (const uint64_t*)ids, (uint64_t*)k1, d2, v1, mm, 0, 64, st);
  cub::DeviceRadixSort::SortPairs(nullptr, tb, (const uint64_t*)k1, (uint64_t*)k2, v1, v2, mm, 0, 63, st);
  const size_t tsz = std::max(ta, tb);
  cudaError_t e = cudaMallocAsync((void**)&k1, 4 * sizeof(int64_t) * (size_t)m + tsz, st);
  if (e != cudaSuccess) return check_cuda(e, "knn sort scratch");
  v1 = k1 + m; k2 = v1 + m; v2 = k2 + m; tmp = (void*)(v2 + m);
  // ids are >= 0 (point_id_base + index) and sort as unsigned; dist2 < 2^63
  size_t t1 = tsz;
  e = cub::DeviceRadixSort::SortPairs(tmp, t1, (const uint64_t*)ids, (uint64_t*)k1, d2, v1, mm, 0, 64, st);
  count_launch();
  if (e == cudaSuccess) {
    size_t t2 = tsz;
    e = cub::DeviceRadixSort::SortPairs(tmp, t2, (const uint64_t*)v1, (uint64_t*)k2, k1, v2, mm, 0, 63, st);
    count_launch();
  }
  const int64_t kk = std::min(k, m);
  if (e == cudaSuccess) {
    k_copy_topk<<<(int)std::min<int64_t>((kk + 255) / 256, 1024), 256, 0, st>>>(v2, k2, kk, out_ids, out_d2);
    count_launch();
    e = cudaGetLastError();
  }
  cudaFreeAsync(k1, st);
  return check_cuda(e, "knn top-k");
}

}  // namespace spade
