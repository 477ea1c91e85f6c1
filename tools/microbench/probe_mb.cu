// Design microbenchmark (not product code): what does a point probe cost on B200?
// Measures, over a 1 G-point int2 stream (8 GB, >> L2):
//   stream   : LDG.128 streaming read only (the roofline for the probe)
//   u8priv   : + random LDS.U16 lookup in a 128 KB smem "coarse canvas" + per-thread u8 counters
//   smatom   : + lookup + smem atomicAdd into u32 bins
//   match    : + lookup + __match_any_sync aggregated smem atomics
//   l2gather : + lookup; "mixed" coarse entries (fraction f) gather a 4 B fine pixel from a 64 MB table
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o probe_mb probe_mb.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

static constexpr int T = 256;          // threads per CTA
static constexpr int U = 4;            // 32-B vectors per thread per iteration (16 points)
static constexpr int NB = 260;         // bins
static constexpr int CW = 256;         // coarse grid 256x256 u16 = 128 KB

struct int8v { int4 a, b; };
// 256-bit load (sm_100: LDG.E.256), streaming hints: bypass L1, evict-first in L2
__device__ __forceinline__ int8v ldg_stream(const int8v* p) {
  int8v r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r.a.x), "=r"(r.a.y), "=r"(r.a.z), "=r"(r.a.w), "=r"(r.b.x), "=r"(r.b.y), "=r"(r.b.z), "=r"(r.b.w) : "l"(p));
  return r;
}

__global__ void gen_points(int2* p, long long n, unsigned long long seed) {
  long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  for (; i < n; i += (long long)gridDim.x * blockDim.x) {
    unsigned long long z = seed + (unsigned long long)i * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    p[i] = make_int2((int)(z & 0xFFFFFF), (int)((z >> 24) & 0xFFFFFF));
  }
}

template <int MODE>
__global__ void __launch_bounds__(T, 1)
probe(const int8v* __restrict__ pts, long long nvec, const uint16_t* __restrict__ gcoarse,
      const int* __restrict__ fine, unsigned long long* __restrict__ out) {
  extern __shared__ __align__(16) unsigned char smem[];
  uint16_t* coarse = (uint16_t*)smem;                         // 128 KB
  uint32_t* hist = (uint32_t*)(smem + CW * CW * 2);           // NB * (T/4+1) words (u8 private) or NB u32
  const int tid = threadIdx.x;
  if (MODE >= 1) {
    for (int i = tid; i < CW * CW / 8; i += T) ((int4*)coarse)[i] = ((const int4*)gcoarse)[i];
    int hw = (MODE == 1) ? NB * (T / 4 + 1) : NB;
    for (int i = tid; i < hw; i += T) hist[i] = 0;
  }
  __syncthreads();
  unsigned long long acc = 0;
  const long long chunk = (long long)T * U;
  int iters = 0;
  for (long long base = (long long)blockIdx.x * chunk; base < nvec; base += (long long)gridDim.x * chunk) {
    int8v v[U];
#pragma unroll
    for (int k = 0; k < U; ++k) {
      long long idx = base + k * T + tid;
      if (idx < nvec) v[k] = ldg_stream(pts + idx); else { v[k].a = make_int4(0,0,0,0); v[k].b = v[k].a; }
    }
#pragma unroll
    for (int k = 0; k < U; ++k) {
#pragma unroll
      for (int h = 0; h < 4; ++h) {
        int x = h == 0 ? v[k].a.x : h == 1 ? v[k].a.z : h == 2 ? v[k].b.x : v[k].b.z;
        int y = h == 0 ? v[k].a.y : h == 1 ? v[k].a.w : h == 2 ? v[k].b.y : v[k].b.w;
        if (MODE == 0) { acc += (unsigned)(x ^ y); continue; }
        unsigned c = coarse[((unsigned)y >> 16) * CW + ((unsigned)x >> 16)];
        if (MODE == 4) {
          if (c == 0xFFFF) c = (unsigned)__ldg(fine + (((unsigned)y >> 12) << 12) + ((unsigned)x >> 12)) % NB;
        } else if (c >= NB) c = 0;
        if (MODE == 1 || MODE == 4) {
          unsigned char* h8 = (unsigned char*)hist;
          int w = c * (T / 4 + 1) + (tid >> 2);
          h8[w * 4 + (tid & 3)] += 1;
        } else if (MODE == 2) {
          atomicAdd(&hist[c], 1u);
        } else if (MODE == 3) {
          unsigned m = __match_any_sync(0xffffffffu, c);
          if ((threadIdx.x & 31) == __ffs(m) - 1) atomicAdd(&hist[c], (unsigned)__popc(m));
        }
      }
    }
    if (MODE == 1 || MODE == 4) {
      if (++iters == 15) {   // flush u8 counters (<= 240 increments each)
        iters = 0;
        __syncthreads();
        for (int b = tid; b < NB; b += T) {
          unsigned s = 0;
          uint32_t* row = hist + b * (T / 4 + 1);
#pragma unroll 8
          for (int q = 0; q < T / 4; ++q) { s = __dp4a(row[q], 0x01010101u, s); row[q] = 0; }
          acc += s;
        }
        __syncthreads();
      }
    }
  }
  if (MODE == 1 || MODE == 4) {
    __syncthreads();
    for (int b = tid; b < NB; b += T) {
      unsigned s = 0; uint32_t* row = hist + b * (T / 4 + 1);
      for (int q = 0; q < T / 4; ++q) s = __dp4a(row[q], 0x01010101u, s);
      acc += s;
    }
  } else if (MODE == 2 || MODE == 3) {
    __syncthreads();
    for (int b = tid; b < NB; b += T) acc += hist[b];
  }
  atomicAdd(out, acc);
}

template <int MODE>
float run(const int8v* pts, long long nvec, const uint16_t* coarse, const int* fine, unsigned long long* out,
          int grid, unsigned long long* result) {
  size_t smem = 0;
  if (MODE >= 1) smem = CW * CW * 2 + ((MODE == 1 || MODE == 4) ? NB * (T / 4 + 1) * 4 : NB * 4);
  CK(cudaFuncSetAttribute(probe<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int w = 0; w < 3; ++w) probe<MODE><<<grid, T, smem>>>(pts, nvec, coarse, fine, out);
  CK(cudaDeviceSynchronize());
  const int reps = 10;
  float best = 1e30f, tot = 0;
  for (int r = 0; r < reps; ++r) {
    CK(cudaMemset(out, 0, 8));
    cudaEventRecord(a);
    probe<MODE><<<grid, T, smem>>>(pts, nvec, coarse, fine, out);
    cudaEventRecord(b); CK(cudaEventSynchronize(b));
    float ms; cudaEventElapsedTime(&ms, a, b); tot += ms; if (ms < best) best = ms;
  }
  CK(cudaMemcpy(result, out, 8, cudaMemcpyDeviceToHost));
  return tot / reps;
}

int main(int argc, char** argv) {
  long long n = argc > 1 ? atoll(argv[1]) : (1ll << 30);
  double mixed_frac = argc > 2 ? atof(argv[2]) : 0.35;
  int dev; CK(cudaGetDevice(&dev)); cudaDeviceProp pr; CK(cudaGetDeviceProperties(&pr, dev));
  int sms = pr.multiProcessorCount;
  printf("device %s SMs %d L2 %d MB\n", pr.name, sms, pr.l2CacheSize >> 20);
  int2* pts; CK(cudaMalloc(&pts, n * 8));
  gen_points<<<sms * 8, 256>>>(pts, n, 12345);
  std::vector<uint16_t> hc(CW * CW);
  srand(7);
  for (auto& c : hc) c = ((double)rand() / RAND_MAX < mixed_frac) ? 0xFFFF : (uint16_t)(rand() % NB);
  uint16_t* dc; CK(cudaMalloc(&dc, hc.size() * 2)); CK(cudaMemcpy(dc, hc.data(), hc.size() * 2, cudaMemcpyHostToDevice));
  int* fine; CK(cudaMalloc(&fine, 4096ll * 4096 * 4)); CK(cudaMemset(fine, 0x11, 4096ll * 4096 * 4));
  unsigned long long* out; CK(cudaMalloc(&out, 8));
  CK(cudaDeviceSynchronize());
  long long nvec = n / 4;
  unsigned long long res;
  double gb = n * 8.0 / 1e9;
  for (int gm : {1, 2, 4}) {
    int grid = sms * gm;
    float t0 = run<0>((int8v*)pts, nvec, dc, fine, out, grid, &res);
    printf("grid %d stream   : %.3f ms  %.1f GB/s  %.3e pts/s\n", grid, t0, gb / t0 * 1e3, n / t0 * 1e3);
    if (gm > 1) continue;  // smem kernels need 1 CTA/SM
    float t1 = run<1>((int8v*)pts, nvec, dc, fine, out, grid, &res);
    printf("grid %d u8priv   : %.3f ms  %.1f GB/s  %.3e pts/s  (sum %llu)\n", grid, t1, gb / t1 * 1e3, n / t1 * 1e3, res);
    float t2 = run<2>((int8v*)pts, nvec, dc, fine, out, grid, &res);
    printf("grid %d smatom   : %.3f ms  %.1f GB/s  %.3e pts/s  (sum %llu)\n", grid, t2, gb / t2 * 1e3, n / t2 * 1e3, res);
    float t3 = run<3>((int8v*)pts, nvec, dc, fine, out, grid, &res);
    printf("grid %d match    : %.3f ms  %.1f GB/s  %.3e pts/s  (sum %llu)\n", grid, t3, gb / t3 * 1e3, n / t3 * 1e3, res);
    float t4 = run<4>((int8v*)pts, nvec, dc, fine, out, grid, &res);
    printf("grid %d l2gather : %.3f ms  %.1f GB/s  %.3e pts/s  (sum %llu, mixed %.2f)\n", grid, t4, gb / t4 * 1e3, n / t4 * 1e3, res, mixed_frac);
  }
  return 0;
}
