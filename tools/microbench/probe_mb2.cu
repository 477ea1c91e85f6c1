// Design microbenchmark #2 (not product code). Isolates the costs of a point probe on B200.
// Stream of 1 G uniform int2 points (8 GB) read with 256-bit loads; per point:
//   LOOKUP : random LDS.U16 into a smem coarse table (CW x CW)
//   HIST   : 0 none, 1 smem atomicAdd (u32 bins), 2 warp-private u32 bins (8 copies) atomics
//   GATHER : "mixed" coarse entries gather 4 B from a global fine table (FMASK+1 ints), phased:
//            all lookups of the 16-point batch first, then all gathers, then all histogram ops.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o probe_mb2 probe_mb2.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)
static constexpr int NB = 260;
struct int8v { int4 a, b; };
__device__ __forceinline__ int8v ldg_stream(const int8v* p) {
  int8v r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r.a.x), "=r"(r.a.y), "=r"(r.a.z), "=r"(r.a.w), "=r"(r.b.x), "=r"(r.b.y), "=r"(r.b.z), "=r"(r.b.w) : "l"(p));
  return r;
}
__device__ __forceinline__ int ldg_keep(const int* p) {
  int r; uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  asm volatile("ld.global.nc.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol)); return r;
}
__global__ void gen_points(int2* p, long long n, unsigned long long seed) {
  long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  for (; i < n; i += (long long)gridDim.x * blockDim.x) {
    unsigned long long z = seed + (unsigned long long)i * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    p[i] = make_int2((int)(z & 0xFFFFFF), (int)((z >> 24) & 0xFFFFFF));
  }
}

template <int T, int CWL2, int LOOKUP, int HIST, int GATHER>
__global__ void __launch_bounds__(T)
probe(const int8v* __restrict__ pts, long long nvec, const uint16_t* __restrict__ gcoarse,
      const int* __restrict__ fine, unsigned fmask, unsigned long long* __restrict__ out) {
  constexpr int CW = 1 << CWL2, U = 4;
  extern __shared__ __align__(16) unsigned char smem[];
  uint16_t* coarse = (uint16_t*)smem;
  uint32_t* hist = (uint32_t*)(smem + (LOOKUP ? CW * CW * 2 : 0));
  constexpr int NCOPY = HIST == 2 ? 8 : 1;
  const int tid = threadIdx.x;
  if (LOOKUP) for (int i = tid; i < CW * CW / 8; i += T) ((int4*)coarse)[i] = ((const int4*)gcoarse)[i];
  if (HIST) for (int i = tid; i < NB * NCOPY; i += T) hist[i] = 0;
  __syncthreads();
  uint32_t* myhist = hist + (HIST == 2 ? (tid >> 5) % NCOPY * NB : 0);
  unsigned long long acc = 0;
  const long long chunk = (long long)T * U;
  for (long long base = (long long)blockIdx.x * chunk; base < nvec; base += (long long)gridDim.x * chunk) {
    int8v v[U];
#pragma unroll
    for (int k = 0; k < U; ++k) {
      long long idx = base + k * T + tid;
      if (idx < nvec) v[k] = ldg_stream(pts + idx); else { v[k].a = make_int4(0,0,0,0); v[k].b = v[k].a; }
    }
    unsigned c[4 * U];
#pragma unroll
    for (int k = 0; k < U; ++k)
#pragma unroll
      for (int h = 0; h < 4; ++h) {
        int x = h == 0 ? v[k].a.x : h == 1 ? v[k].a.z : h == 2 ? v[k].b.x : v[k].b.z;
        int y = h == 0 ? v[k].a.y : h == 1 ? v[k].a.w : h == 2 ? v[k].b.y : v[k].b.w;
        unsigned cc;
        if (LOOKUP) cc = coarse[(((unsigned)y >> (24 - CWL2)) << CWL2) + ((unsigned)x >> (24 - CWL2))];
        else cc = ((unsigned)(x ^ y)) % NB;
        if (GATHER) {
          if (cc == 0xFFFFu) cc = 0x80000000u | ((((unsigned)y >> 12) << 12) + ((unsigned)x >> 12));
        }
        c[4 * k + h] = cc;
      }
    if (GATHER) {
#pragma unroll
      for (int q = 0; q < 4 * U; ++q)
        if (c[q] & 0x80000000u) c[q] = (unsigned)ldg_keep(fine + (c[q] & fmask)) % NB;
    }
#pragma unroll
    for (int q = 0; q < 4 * U; ++q) {
      unsigned b = c[q] >= NB ? 0 : c[q];
      if (HIST) atomicAdd(&myhist[b], 1u); else acc += b;
    }
  }
  if (HIST) {
    __syncthreads();
    for (int b = tid; b < NB * NCOPY; b += T) acc += hist[b];
  }
  atomicAdd(out, acc);
}

template <int T, int CWL2, int LOOKUP, int HIST, int GATHER>
void run(const char* name, const int8v* pts, long long nvec, const uint16_t* coarse, const int* fine, unsigned fmask,
         unsigned long long* out, int grid, double npts) {
  constexpr int CW = 1 << CWL2;
  size_t smem = (LOOKUP ? CW * CW * 2 : 0) + (HIST ? NB * 4 * (HIST == 2 ? 8 : 1) : 0);
  auto kern = probe<T, CWL2, LOOKUP, HIST, GATHER>;
  CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int w = 0; w < 2; ++w) kern<<<grid, T, smem>>>(pts, nvec, coarse, fine, fmask, out);
  CK(cudaDeviceSynchronize());
  const int reps = 8; float tot = 0;
  for (int r = 0; r < reps; ++r) {
    cudaEventRecord(a);
    kern<<<grid, T, smem>>>(pts, nvec, coarse, fine, fmask, out);
    cudaEventRecord(b); CK(cudaEventSynchronize(b));
    float ms; cudaEventElapsedTime(&ms, a, b); tot += ms;
  }
  float t = tot / reps;
  printf("%-34s grid %4d T %4d smem %6zu : %.3f ms %7.1f GB/s %.3e pts/s\n", name, grid, T, smem, t,
         npts * 8 / t / 1e6, npts / t * 1e3);
}

int main(int argc, char** argv) {
  long long n = 1ll << 30;
  int dev; CK(cudaGetDevice(&dev)); cudaDeviceProp pr; CK(cudaGetDeviceProperties(&pr, dev));
  int sms = pr.multiProcessorCount;
  int2* pts; CK(cudaMalloc(&pts, n * 8));
  gen_points<<<sms * 8, 256>>>(pts, n, 12345);
  auto mkcoarse = [&](int cw, double mixed) {
    std::vector<uint16_t> hc((size_t)cw * cw);
    srand(7);
    for (auto& c : hc) c = ((double)rand() / RAND_MAX < mixed) ? 0xFFFF : (uint16_t)(rand() % NB);
    uint16_t* dc; CK(cudaMalloc(&dc, hc.size() * 2)); CK(cudaMemcpy(dc, hc.data(), hc.size() * 2, cudaMemcpyHostToDevice));
    return dc;
  };
  uint16_t* c256_0 = mkcoarse(256, 0.0), *c256_10 = mkcoarse(256, 0.10), *c256_35 = mkcoarse(256, 0.35);
  uint16_t* c256_100 = mkcoarse(256, 1.0);
  uint16_t* c128_0 = mkcoarse(128, 0.0);
  int* fine; CK(cudaMalloc(&fine, 4096ll * 4096 * 4)); CK(cudaMemset(fine, 0x11, 4096ll * 4096 * 4));
  unsigned long long* out; CK(cudaMalloc(&out, 8));
  CK(cudaDeviceSynchronize());
  long long nvec = n / 4; double np = (double)n;
  const int8v* P = (const int8v*)pts;
  unsigned m64 = (1u << 24) - 1, m16 = (1u << 22) - 1, m4 = (1u << 20) - 1;
  run<256, 8, 0, 0, 0>("stream(+hash)", P, nvec, c256_0, fine, m64, out, sms * 2, np);
  run<512, 8, 0, 0, 0>("stream(+hash)", P, nvec, c256_0, fine, m64, out, sms * 2, np);
  run<256, 8, 1, 0, 0>("lookup only cw256", P, nvec, c256_0, fine, m64, out, sms, np);
  run<512, 8, 1, 0, 0>("lookup only cw256", P, nvec, c256_0, fine, m64, out, sms, np);
  run<1024, 8, 1, 0, 0>("lookup only cw256", P, nvec, c256_0, fine, m64, out, sms, np);
  run<256, 7, 1, 0, 0>("lookup only cw128", P, nvec, c128_0, fine, m64, out, sms * 4, np);
  run<256, 8, 0, 1, 0>("hash+smatom", P, nvec, c256_0, fine, m64, out, sms * 4, np);
  run<256, 8, 0, 2, 0>("hash+smatom 8 copies", P, nvec, c256_0, fine, m64, out, sms * 4, np);
  run<256, 8, 1, 1, 0>("lookup+smatom cw256", P, nvec, c256_0, fine, m64, out, sms, np);
  run<512, 8, 1, 1, 0>("lookup+smatom cw256", P, nvec, c256_0, fine, m64, out, sms, np);
  run<1024, 8, 1, 1, 0>("lookup+smatom cw256", P, nvec, c256_0, fine, m64, out, sms, np);
  run<512, 8, 1, 2, 0>("lookup+smatom8 cw256", P, nvec, c256_0, fine, m64, out, sms, np);
  run<256, 7, 1, 1, 0>("lookup+smatom cw128 4cta", P, nvec, c128_0, fine, m64, out, sms * 4, np);
  run<512, 8, 1, 0, 1>("lookup+gather 10% 64MB", P, nvec, c256_10, fine, m64, out, sms, np);
  run<512, 8, 1, 0, 1>("lookup+gather 35% 64MB", P, nvec, c256_35, fine, m64, out, sms, np);
  run<512, 8, 1, 0, 1>("lookup+gather 100% 64MB", P, nvec, c256_100, fine, m64, out, sms, np);
  run<512, 8, 1, 0, 1>("lookup+gather 100% 16MB", P, nvec, c256_100, fine, m16, out, sms, np);
  run<512, 8, 1, 0, 1>("lookup+gather 100% 4MB", P, nvec, c256_100, fine, m4, out, sms, np);
  run<512, 8, 1, 0, 1>("lookup+gather 35% 16MB", P, nvec, c256_35, fine, m16, out, sms, np);
  run<512, 8, 1, 1, 1>("lookup+gather35%64MB+smatom", P, nvec, c256_35, fine, m64, out, sms, np);
  run<512, 8, 1, 1, 1>("lookup+gather10%64MB+smatom", P, nvec, c256_10, fine, m64, out, sms, np);
  return 0;
}
