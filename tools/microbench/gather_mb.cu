// Design microbenchmark (not product code): random 4-B / 2-B gathers on B200 through the LSU path
// (ld.global.nc) versus the texture path (tex1Dfetch on a linear-memory texture object), alone
// and next to a 256-bit streaming read (the probe's point stream).  Question: is the L1 data-pipe
// cost of a 32-lane random gather (one wavefront per distinct line on the LSU path) lower through
// the TEX pipe, which the probe leaves idle?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o gather_mb gather_mb.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

struct V8 { int4 a, b; };
__device__ __forceinline__ V8 ld_stream(const V8* p) {
  V8 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r.a.x), "=r"(r.a.y), "=r"(r.a.z), "=r"(r.a.w), "=r"(r.b.x), "=r"(r.b.y), "=r"(r.b.z), "=r"(r.b.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}

// MODE 0: LSU gathers (int32), 1: TEX gathers (int32), 2: LSU u16, 3: TEX u16
// STREAM: also stream one 32-B vector per thread per iteration (4 "points": 4 gathers each)
// frac_mask: a point gathers when (hash & 1023) < fthr (fraction of points that gather)
template <int MODE, bool STREAM>
__global__ void __launch_bounds__(1024, 1) k_gather(const int32_t* __restrict__ a32, const uint16_t* __restrict__ a16,
                                                    cudaTextureObject_t tex, uint32_t nelem, const V8* __restrict__ s,
                                                    uint32_t nvec, uint32_t iters, uint32_t fthr, unsigned long long* out) {
  uint32_t acc = 0;
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x, nt = gridDim.x * blockDim.x;
  for (uint32_t it = 0; it < iters; ++it) {
    uint32_t h[4];
    if (STREAM) {
      const uint32_t vi = (it * nt + tid) % nvec;
      const V8 v = ld_stream(s + vi);
      h[0] = (uint32_t)v.a.x; h[1] = (uint32_t)v.a.z; h[2] = (uint32_t)v.b.x; h[3] = (uint32_t)v.b.z;
    } else {
#pragma unroll
      for (int q = 0; q < 4; ++q) h[q] = (it * nt * 4 + tid * 4 + q) * 2654435761u ^ (it * 0x9E3779B9u);
    }
    uint32_t g[4] = {0, 0, 0, 0};
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if ((h[q] & 1023u) < fthr) {
        const uint32_t idx = (h[q] >> 10) % nelem;
        if (MODE == 0) g[q] = (uint32_t)__ldg(a32 + idx);
        else if (MODE == 1) g[q] = (uint32_t)tex1Dfetch<int>(tex, (int)idx);
        else if (MODE == 2) g[q] = (uint32_t)__ldg(a16 + idx);
        else g[q] = (uint32_t)tex1Dfetch<unsigned short>(tex, (int)idx);
      }
    }
    acc += g[0] ^ g[1] ^ g[2] ^ g[3];
  }
  if (acc == 0x12345678u) atomicAdd(out, 1ull);
}

__global__ void k_fill(uint32_t* p, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) p[i] = hash32((uint32_t)i * 2654435761u + 12345u);
}

int main(int argc, char** argv) {
  const size_t mb = argc > 1 ? atoi(argv[1]) : 64;            // gather table size (MB)
  const uint32_t n32 = (uint32_t)(mb << 18), n16 = (uint32_t)(mb << 19);
  int32_t* a32; uint16_t* a16; V8* s; unsigned long long* out;
  const uint32_t nvec = 1u << 28;                              // 8 GB stream (> L2)
  CK(cudaMalloc(&a32, (size_t)n32 * 4)); CK(cudaMalloc(&a16, (size_t)n16 * 2));
  CK(cudaMalloc(&s, (size_t)nvec * 32)); CK(cudaMalloc(&out, 8));
  CK(cudaMemset(a32, 1, (size_t)n32 * 4)); CK(cudaMemset(a16, 1, (size_t)n16 * 2)); k_fill<<<4096, 256>>>((uint32_t*)s, (size_t)nvec * 8); CK(cudaDeviceSynchronize());
  cudaTextureObject_t t32, t16;
  {
    cudaResourceDesc rd = {}; rd.resType = cudaResourceTypeLinear;
    rd.res.linear.devPtr = a32; rd.res.linear.desc = cudaCreateChannelDesc<int>(); rd.res.linear.sizeInBytes = (size_t)n32 * 4;
    cudaTextureDesc td = {}; td.readMode = cudaReadModeElementType;
    CK(cudaCreateTextureObject(&t32, &rd, &td, nullptr));
    rd.res.linear.devPtr = a16; rd.res.linear.desc = cudaCreateChannelDesc<unsigned short>(); rd.res.linear.sizeInBytes = (size_t)n16 * 2;
    CK(cudaCreateTextureObject(&t16, &rd, &td, nullptr));
  }
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const uint32_t iters = 2048;
  const double pts = (double)sms * 1024 * iters * 4;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  auto run = [&](const char* name, auto kern, cudaTextureObject_t t, uint32_t nel, uint32_t fthr) {
    for (int r = 0; r < 2; ++r) kern<<<sms, 1024>>>(a32, a16, t, nel, s, nvec, iters, fthr, out);
    CK(cudaEventRecord(e0));
    const int reps = 5;
    for (int r = 0; r < reps; ++r) kern<<<sms, 1024>>>(a32, a16, t, nel, s, nvec, iters, fthr, out);
    CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms, e0, e1); ms /= reps;
    printf("%-26s table %4zu MB  gather frac %.2f  %.3f ms  %.2f Gpoints/s  %.2f Ggathers/s\n", name, mb, fthr / 1024.0, ms,
           pts / ms * 1e-6, pts * fthr / 1024.0 / ms * 1e-6);
  };
  for (uint32_t fthr : {1024u, 440u, 184u}) {
    run("lsu32", k_gather<0, false>, t32, n32, fthr);
    run("tex32", k_gather<1, false>, t32, n32, fthr);
    run("lsu16", k_gather<2, false>, t16, n16, fthr);
    run("tex16", k_gather<3, false>, t16, n16, fthr);
    run("lsu32+stream", k_gather<0, true>, t32, n32, fthr);
    run("tex32+stream", k_gather<1, true>, t32, n32, fthr);
    run("lsu16+stream", k_gather<2, true>, t16, n16, fthr);
    run("tex16+stream", k_gather<3, true>, t16, n16, fthr);
  }
  run("stream only", k_gather<0, true>, t32, n32, 0);
  return 0;
}
