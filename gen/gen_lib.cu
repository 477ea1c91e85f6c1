/*
 * gen_lib.cu — libspade_gen.so: host and device drivers for the counter-based point generator
 * in spade_gen.h (input data only; no join arithmetic).  Used by tests, smoke() and bench.py to
 * create device-resident shards (sg_points_device) and bit-identical host samples
 * (sg_points_host / sg_points_at).
 */
#include <cuda_runtime.h>
#include "spade_gen.h"

__global__ void sg_points_kernel(sg_params p, uint64_t seed, uint64_t start, int64_t n, int2* out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int32_t x, y;
        sg_point(&p, seed, start + (uint64_t)i, &x, &y);
        out[i] = make_int2(x, y);
    }
}

extern "C" {

/* Points [start, start+n) into DEVICE buffer out (n x int2), enqueued on `stream`. 0 = ok. */
int sg_points_device(const sg_params* p, uint64_t seed, uint64_t start, int64_t n, int32_t* out, void* stream) {
    if (n <= 0) return 0;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int64_t blocks = (n + 255) / 256;
    if (blocks > (int64_t)sms * 16) blocks = (int64_t)sms * 16;
    sg_points_kernel<<<(int)blocks, 256, 0, (cudaStream_t)stream>>>(*p, seed, start, n, (int2*)out);
    return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

/* Points [start, start+n) into HOST buffer out. */
void sg_points_host(const sg_params* p, uint64_t seed, uint64_t start, int64_t n, int32_t* out) {
    for (int64_t i = 0; i < n; ++i) sg_point(p, seed, start + (uint64_t)i, &out[2 * i], &out[2 * i + 1]);
}

/* Points at arbitrary global indices into HOST buffer out. */
void sg_points_at(const sg_params* p, uint64_t seed, const int64_t* idx, int64_t n, int32_t* out) {
    for (int64_t i = 0; i < n; ++i) sg_point(p, seed, (uint64_t)idx[i], &out[2 * i], &out[2 * i + 1]);
}

int sg_params_size(void) { return (int)sizeof(sg_params); }

}  // extern "C"
