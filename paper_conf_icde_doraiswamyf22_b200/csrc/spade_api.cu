// spade_api.cu — the C ABI (include/spade.h): argument validation, status codes, thread-local
// error detail, launch accounting, the capacity protocol of the Map operator (PAPER.md P:167-175:
// 1-pass Map when n_max fits, else count first and retry) and the host-resident streaming join.
#include <cstdarg>
#include <cstdlib>
#include <string>
#include <cstdio>
#include <cstring>
#include <atomic>
#include <algorithm>
#include <vector>
#include <nvtx3/nvToolsExt.h>
#include "spade_internal.cuh"

namespace spade {

// NVTX range for the duration of one entry point (visible in nsys / ncu --nvtx)
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

int build_canvas(const int32_t*, const int64_t*, const int64_t*, int32_t, const spade_canvas_params*, cudaStream_t,
                 spade_canvas**);
int build_disk_canvas(const int32_t*, const int64_t*, int32_t, const spade_canvas_params*, cudaStream_t, spade_canvas**);
int canvas_checksum(const spade_canvas*, uint64_t*, cudaStream_t);
int join_polygons(const int32_t*, const int64_t*, const int64_t*, int32_t, const int32_t*, const int64_t*, const int64_t*,
                  int32_t, const spade_canvas_params*, int32_t*, int32_t*, int64_t, int64_t*, cudaStream_t);

namespace {
thread_local char g_err[512] = "";
std::atomic<int64_t> g_launches{0};
}  // namespace

int set_error(int code, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
  return code;
}

int check_cuda(cudaError_t e, const char* what) {
  if (e == cudaSuccess) return SPADE_OK;
  if (e == cudaErrorMemoryAllocation) return set_error(SPADE_ERR_OOM, "%s: %s", what, cudaGetErrorString(e));
  return set_error(SPADE_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

void count_launch(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

int device_sm_count() {
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms <= 0) sms = 148;
  return sms;
}

// Streams and events of the host-resident calls, created once per thread and device and reused
// (a call used to create 2-3 streams and 4-8 events and cudaMalloc its staging buffers; those now
// come from the stream-ordered pool).
struct HostStreams {
  bool ok = false;
  cudaStream_t s[3] = {};
  cudaEvent_t ev[8] = {};
};
static HostStreams* host_streams() {
  static thread_local HostStreams hs[16];
  int dev = 0;
  cudaGetDevice(&dev);
  HostStreams& h = hs[dev & 15];
  if (!h.ok) {
    for (cudaStream_t& st : h.s)
      if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess) return nullptr;
    for (cudaEvent_t& e : h.ev)
      if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return nullptr;
    h.ok = true;
  }
  return &h;
}

static int check_points(const spade_canvas* c, const int32_t* xy, int64_t n, const char* fn) {
  if (!c) return set_error(SPADE_ERR_INVALID_ARG, "%s: canvas is NULL", fn);
  if (n < 0) return set_error(SPADE_ERR_INVALID_ARG, "%s: negative n", fn);
  if (n > 0 && !xy) return set_error(SPADE_ERR_INVALID_ARG, "%s: xy is NULL", fn);
  if (n > 0 && ((uintptr_t)xy & 7)) return set_error(SPADE_ERR_INVALID_ARG, "%s: xy must be 8-byte aligned", fn);
  return SPADE_OK;
}

}  // namespace spade

namespace spade {
// Map with capacity: one device counter; the kernel writes results below `capacity` and counts
// all of them; the host reads the total (P:173 1-pass, P:175 2-pass on overflow).
template <class F>
int run_with_capacity(int64_t capacity, int64_t* n_out, cudaStream_t st, const char* fn, F launch) {
  if (!n_out) return set_error(SPADE_ERR_INVALID_ARG, "%s: n_out is NULL", fn);
  if (capacity < 0) return set_error(SPADE_ERR_INVALID_ARG, "%s: negative capacity", fn);
  unsigned long long* d_total = nullptr;
  cudaError_t e = cudaMallocAsync((void**)&d_total, sizeof(unsigned long long), st);
  if (e != cudaSuccess) return check_cuda(e, fn);
  e = cudaMemsetAsync(d_total, 0, sizeof(unsigned long long), st);
  int rc = e == cudaSuccess ? launch(d_total) : check_cuda(e, fn);
  // the count comes back through a pinned word (one per thread, allocated once): a DMA instead of a
  // staged copy into pageable memory
  static thread_local unsigned long long* pinned = nullptr;
  if (!pinned && cudaMallocHost((void**)&pinned, sizeof(unsigned long long)) != cudaSuccess) {
    pinned = nullptr;
    cudaGetLastError();
  }
  unsigned long long h = 0;
  if (rc == SPADE_OK) {
    e = cudaMemcpyAsync(pinned ? pinned : &h, d_total, sizeof(h), cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) rc = check_cuda(e, fn);
    else if (pinned) h = *pinned;
  }
  cudaFreeAsync(d_total, st);
  if (rc != SPADE_OK) return rc;
  *n_out = (int64_t)h;
  if ((int64_t)h > capacity)
    return set_error(SPADE_ERR_CAPACITY, "%s: %lld results exceed capacity %lld", fn, (long long)h, (long long)capacity);
  return SPADE_OK;
}

}  // namespace spade

using namespace spade;

namespace spade {
static int env_int(const char* name, int dflt) {
  const char* e = getenv(name);
  return e ? atoi(e) : dflt;
}
Options& options() {
  static Options o{env_int("SPADE_DEFER", 0), env_int("SPADE_COUNT_GLOBAL", 0), env_int("SPADE_GLOBAL_QUEUE", 0),
                   env_int("SPADE_CACHE_SLOTS", 4096), env_int("SPADE_COOP", 0), env_int("SPADE_DEBUG_DEFER", 0),
                   env_int("SPADE_PIPE", -1), env_int("SPADE_DEFER_XY", 0), env_int("SPADE_L2_FRAC_PCT", 100), env_int("SPADE_MULTI_AGG", 1), env_int("SPADE_K_AGG", -1),
                   (int64_t)1 << 25, (1ll << 31) - 64, 4096, env_int("SPADE_FINE16", 1),
                   env_int("SPADE_STAGE_EVENTS", 0), env_int("SPADE_TMA", 0), env_int("SPADE_SMEM_PAD_KB", 0),
                   env_int("SPADE_TMA_SLACK_KB", 0), env_int("SPADE_PIPE_NOTILE", 0),
                   env_int("SPADE_HIST_COPIES_MAX", 16), env_int("SPADE_IDX_QUEUE", -1)};
  return o;
}
}  // namespace spade

extern "C" {

int spade_build_canvas(const int32_t* ring_xy, const int64_t* ring_off, const int64_t* poly_ring_off,
                       int32_t num_polys, const spade_canvas_params* prm, spade_stream_t stream, spade_canvas** out) {
  if (!out) return set_error(SPADE_ERR_INVALID_ARG, "spade_build_canvas: out is NULL");
  *out = nullptr;
  NvtxRange nv("spade_build_canvas");
  return build_canvas(ring_xy, ring_off, poly_ring_off, num_polys, prm, (cudaStream_t)stream, out);
}

int spade_build_disk_canvas(const int32_t* center_xy, const int64_t* r2, int32_t num_disks,
                            const spade_canvas_params* prm, spade_stream_t stream, spade_canvas** out) {
  if (!out) return set_error(SPADE_ERR_INVALID_ARG, "spade_build_disk_canvas: out is NULL");
  *out = nullptr;
  NvtxRange nv("spade_build_disk_canvas");
  return build_disk_canvas(center_xy, r2, num_disks, prm, (cudaStream_t)stream, out);
}

void spade_canvas_free(spade_canvas* c) {
  if (!c) return;
  DeviceGuard dg(c->device);
  cudaDeviceSynchronize();
  // every canvas array comes from the stream-ordered pool (spade_build_canvas): back to the pool
  for (void* p : {(void*)c->fine, (void*)c->fine16, (void*)c->cfine, (void*)c->coarse, (void*)c->recs, (void*)c->blob,
                  (void*)c->sets, (void*)c->set_rng, (void*)c->kbits, (void*)c->d_dev})
    if (p) cudaFreeAsync(p, 0);
  cudaStreamSynchronize(0);
  cudaGetLastError();
  delete c;
}

int spade_canvas_info(const spade_canvas* c, int32_t* W, int32_t* H, int32_t* log2_pixel, int32_t* Wc, int32_t* Hc,
                      int32_t* log2_tile, int64_t* num_runs, int64_t* num_run_edges, double* mixed_tile_frac) {
  if (!c) return set_error(SPADE_ERR_INVALID_ARG, "spade_canvas_info: canvas is NULL");
  if (W) *W = c->empty ? 0 : c->d.W;
  if (H) *H = c->empty ? 0 : c->d.H;
  if (log2_pixel) *log2_pixel = c->empty ? 0 : c->d.s;
  if (Wc) *Wc = c->empty ? 0 : c->d.Wc;
  if (Hc) *Hc = c->empty ? 0 : c->d.Hc;
  if (log2_tile) *log2_tile = c->empty ? 0 : c->d.b;
  if (num_runs) *num_runs = c->num_records;
  if (num_run_edges) *num_run_edges = c->num_run_edges;
  if (mixed_tile_frac) *mixed_tile_frac = c->mixed_tile_frac;
  return SPADE_OK;
}

int spade_join_polygons(const int32_t* ring_xy1, const int64_t* ring_off1, const int64_t* poly_ring_off1, int32_t num_polys1,
                        const int32_t* ring_xy2, const int64_t* ring_off2, const int64_t* poly_ring_off2, int32_t num_polys2,
                        const spade_canvas_params* prm, int32_t* out_a, int32_t* out_b, int64_t capacity, int64_t* n_out,
                        spade_stream_t stream) {
  if (!n_out) return set_error(SPADE_ERR_INVALID_ARG, "spade_join_polygons: n_out is NULL");
  NvtxRange nv("spade_join_polygons");
  return join_polygons(ring_xy1, ring_off1, poly_ring_off1, num_polys1, ring_xy2, ring_off2, poly_ring_off2, num_polys2,
                       prm, out_a, out_b, capacity, n_out, (cudaStream_t)stream);
}

int spade_canvas_build_times(const spade_canvas* c, float* ms, int32_t cap) {
  if (!c || (cap > 0 && !ms) || cap < 0) return set_error(SPADE_ERR_INVALID_ARG, "spade_canvas_build_times: bad arguments");
  for (int i = 0; i < c->num_stages && i < cap; ++i) ms[i] = c->stage_ms[i];
  return c->num_stages;
}

const char* spade_canvas_build_stage_name(int32_t i) {
  return i >= 0 && i < kBuildStages ? kBuildStageNames[i] : nullptr;
}

int spade_canvas_checksum(const spade_canvas* c, uint64_t* out, spade_stream_t stream) {
  if (!c || !out) return set_error(SPADE_ERR_INVALID_ARG, "spade_canvas_checksum: NULL argument");
  DeviceGuard dg(c->device);
  return canvas_checksum(c, out, (cudaStream_t)stream);
}

int spade_join_count(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t* counts, spade_stream_t stream) {
  int rc = check_points(c, xy, n, "spade_join_count");
  if (rc) return rc;
  if (c->d.num_polys > 0 && !counts) return set_error(SPADE_ERR_INVALID_ARG, "spade_join_count: counts is NULL");
  DeviceGuard dg(c->device);
  NvtxRange nv("spade_join_count");
  return launch_count(c, xy, n, counts, (cudaStream_t)stream);
}

int spade_select(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t point_id_base, int64_t* out_ids,
                 int64_t capacity, int64_t* n_out, spade_stream_t stream) {
  int rc = check_points(c, xy, n, "spade_select");
  if (rc) return rc;
  if (capacity > 0 && !out_ids) return set_error(SPADE_ERR_INVALID_ARG, "spade_select: out_ids is NULL");
  DeviceGuard dg(c->device);
  NvtxRange nv("spade_select");
  return run_with_capacity(capacity, n_out, (cudaStream_t)stream, "spade_select", [&](unsigned long long* t) {
    return launch_select(c, xy, n, point_id_base, out_ids, capacity, t, (cudaStream_t)stream);
  });
}

int spade_join_pairs(const spade_canvas* c, const int32_t* xy, int64_t n, int64_t point_id_base, int64_t* out_point_ids,
                     int32_t* out_poly_ids, int64_t capacity, int64_t* n_out, spade_stream_t stream) {
  int rc = check_points(c, xy, n, "spade_join_pairs");
  if (rc) return rc;
  if (capacity > 0 && (!out_point_ids || !out_poly_ids))
    return set_error(SPADE_ERR_INVALID_ARG, "spade_join_pairs: output arrays are NULL");
  DeviceGuard dg(c->device);
  NvtxRange nv("spade_join_pairs");
  return run_with_capacity(capacity, n_out, (cudaStream_t)stream, "spade_join_pairs", [&](unsigned long long* t) {
    return launch_pairs(c, xy, n, point_id_base, out_point_ids, out_poly_ids, capacity, t, (cudaStream_t)stream);
  });
}

// Host-resident points: chunks of kChunk points are copied into two device staging buffers on a
// copy stream while the probe consumes the previous chunk on a compute stream (P:480 proposes
// exactly this pipelining of I/O with GPU work).
int spade_join_count_host(const spade_canvas* c, const int32_t* xy_host, int64_t n, int64_t* counts_host,
                          spade_stream_t stream) {
  int rc = check_points(c, xy_host, n, "spade_join_count_host");
  if (rc) return rc;
  const int P = c->d.num_polys;
  if (P > 0 && !counts_host) return set_error(SPADE_ERR_INVALID_ARG, "spade_join_count_host: counts_host is NULL");
  if (n == 0 || P == 0) return SPADE_OK;
  DeviceGuard dg(c->device);
  NvtxRange nv("spade_join_count_host");
  cudaStream_t st = (cudaStream_t)stream;
  const int64_t kChunk = options().host_chunk;  // default 32 Mi points = 256 MiB per staging buffer
  const int64_t chunk = std::min(kChunk, n);
  int32_t* stage[2] = {nullptr, nullptr};
  int64_t* d_counts = nullptr;
  HostStreams* hs = host_streams();
  if (!hs) return set_error(SPADE_ERR_CUDA, "spade_join_count_host: stream setup failed");
  keep_pool_memory();
  cudaStream_t cs = hs->s[0], ks = hs->s[1];
  cudaEvent_t copied[2] = {hs->ev[0], hs->ev[1]}, consumed[2] = {hs->ev[2], hs->ev[3]};
  cudaError_t e = cudaSuccess;
  auto cleanup = [&]() {
    cudaStreamSynchronize(ks);
    cudaStreamSynchronize(cs);
    for (int i = 0; i < 2; ++i)
      if (stage[i]) cudaFreeAsync(stage[i], st);
    if (d_counts) cudaFreeAsync(d_counts, st);
  };
#define HTRY(call, what) do { e = (call); if (e != cudaSuccess) { int r_ = check_cuda(e, what); cleanup(); return r_; } } while (0)
  HTRY(cudaMallocAsync((void**)&stage[0], chunk * 8, st), "staging");
  HTRY(cudaMallocAsync((void**)&stage[1], chunk * 8, st), "staging");
  HTRY(cudaMallocAsync((void**)&d_counts, sizeof(int64_t) * P, st), "counts");
  // order after prior work on the caller's stream
  HTRY(cudaEventRecord(consumed[0], st), "event");
  HTRY(cudaStreamWaitEvent(cs, consumed[0], 0), "wait");
  HTRY(cudaStreamWaitEvent(ks, consumed[0], 0), "wait");
  HTRY(cudaMemsetAsync(d_counts, 0, sizeof(int64_t) * P, ks), "memset");
  int64_t k = 0;
  for (int64_t off = 0; off < n; off += chunk, ++k) {
    const int b = (int)(k & 1);
    const int64_t m = std::min(chunk, n - off);
    if (k >= 2) HTRY(cudaStreamWaitEvent(cs, consumed[b], 0), "wait");
    HTRY(cudaMemcpyAsync(stage[b], xy_host + 2 * off, m * 8, cudaMemcpyHostToDevice, cs), "H2D");
    HTRY(cudaEventRecord(copied[b], cs), "event");
    HTRY(cudaStreamWaitEvent(ks, copied[b], 0), "wait");
    rc = launch_count(c, stage[b], m, d_counts, ks);
    if (rc != SPADE_OK) { cleanup(); return rc; }
    HTRY(cudaEventRecord(consumed[b], ks), "event");
  }
  std::vector<int64_t> h(P);
  HTRY(cudaMemcpyAsync(h.data(), d_counts, sizeof(int64_t) * P, cudaMemcpyDeviceToHost, ks), "D2H");
  HTRY(cudaStreamSynchronize(ks), "sync");
  for (int p = 0; p < P; ++p) counts_host[p] += h[p];
  // make the caller's stream observe completion
  HTRY(cudaEventRecord(consumed[0], ks), "event");
  HTRY(cudaStreamWaitEvent(st, consumed[0], 0), "wait");
  cleanup();
  return SPADE_OK;
#undef HTRY
}

// Host-resident points, SELECT / PAIRS: the Map of P:167-175 applied chunk by chunk to a point
// stream that lives on the host (NEXT(3)).  Three streams overlap:
//   cs  H2D of chunk k+1 into staging buffer (k+1)&1
//   ks  probe of chunk k into device result buffer k&1, then its result count D2H (pinned word)
//   ds  D2H of chunk k-1's results into the caller's host arrays at the running offset
// The host waits only on chunk k-1's count, after chunk k's probe is already enqueued.  A chunk
// whose results exceed its device buffer (possible for PAIRS with overlapping polygons) is re-run
// with a buffer of the reported size (the 2-pass Map).  Results beyond `capacity` are
// counted but not copied; the call then returns SPADE_ERR_CAPACITY with *n_out = the total.
// Output order: chunk order; within a chunk unspecified (as the device calls).
static int map_host(const spade_canvas* c, const int32_t* xy_host, int64_t n, int64_t base, int64_t* out_ids,
                    int32_t* out_polys, int64_t capacity, int64_t* n_out, cudaStream_t st, const char* fn) {
  DeviceGuard dg(c->device);
  NvtxRange nv(fn);
  const bool pairs = out_polys != nullptr || std::string(fn) == "spade_join_pairs_host";
  const int64_t chunk = std::min(options().host_chunk, n);
  int32_t* stage[2] = {nullptr, nullptr};
  int64_t* d_ids[2] = {nullptr, nullptr};
  int32_t* d_polys[2] = {nullptr, nullptr};
  int64_t cap_b[2] = {chunk, chunk};
  unsigned long long* d_tot = nullptr;   // [2] device result counters
  unsigned long long* h_tot = nullptr;   // [2] pinned copies
  HostStreams* hs = host_streams();
  if (!hs) return set_error(SPADE_ERR_CUDA, "%s: stream setup failed", fn);
  keep_pool_memory();
  cudaStream_t cs = hs->s[0], ks = hs->s[1], ds = hs->s[2];
  cudaEvent_t copied[2] = {hs->ev[0], hs->ev[1]}, consumed[2] = {hs->ev[2], hs->ev[3]},
              probed[2] = {hs->ev[4], hs->ev[5]}, drained[2] = {hs->ev[6], hs->ev[7]};
  cudaError_t e = cudaSuccess;
  auto cleanup = [&]() {
    for (cudaStream_t s : {ks, cs, ds}) cudaStreamSynchronize(s);
    for (int i = 0; i < 2; ++i) {
      if (stage[i]) cudaFreeAsync(stage[i], st);
      if (d_ids[i]) cudaFreeAsync(d_ids[i], st);
      if (d_polys[i]) cudaFreeAsync(d_polys[i], st);
    }
    if (d_tot) cudaFreeAsync(d_tot, st);
    if (h_tot) cudaFreeHost(h_tot);
  };
#define MTRY(call, what) do { e = (call); if (e != cudaSuccess) { int r_ = check_cuda(e, what); cleanup(); return r_; } } while (0)
#define MRC(expr) do { int r_ = (expr); if (r_ != SPADE_OK) { cleanup(); return r_; } } while (0)
  for (int i = 0; i < 2; ++i) {
    MTRY(cudaMallocAsync((void**)&stage[i], chunk * 8, st), "staging");
    MTRY(cudaMallocAsync((void**)&d_ids[i], chunk * 8, st), "result buffer");
    if (pairs) MTRY(cudaMallocAsync((void**)&d_polys[i], chunk * 4, st), "result buffer");
  }
  MTRY(cudaMallocAsync((void**)&d_tot, 2 * sizeof(unsigned long long), st), "counter");
  MTRY(cudaHostAlloc(&h_tot, 2 * sizeof(unsigned long long), cudaHostAllocDefault), "pinned counter");
  MTRY(cudaEventRecord(consumed[0], st), "event");   // order after prior work on the caller's stream
  for (cudaStream_t s : {cs, ks, ds}) MTRY(cudaStreamWaitEvent(s, consumed[0], 0), "wait");

  auto probe = [&](int b, int64_t off, int64_t m) -> int {
    cudaError_t e2 = cudaMemsetAsync(d_tot + b, 0, sizeof(unsigned long long), ks);
    if (e2 != cudaSuccess) return check_cuda(e2, fn);
    int rc = pairs ? launch_pairs(c, stage[b], m, base + off, d_ids[b], d_polys[b], cap_b[b], d_tot + b, ks)
                   : launch_select(c, stage[b], m, base + off, d_ids[b], cap_b[b], d_tot + b, ks);
    if (rc != SPADE_OK) return rc;
    e2 = cudaMemcpyAsync(h_tot + b, d_tot + b, sizeof(unsigned long long), cudaMemcpyDeviceToHost, ks);
    if (e2 == cudaSuccess) e2 = cudaEventRecord(probed[b], ks);
    return check_cuda(e2, fn);
  };
  int64_t total = 0;
  // drain chunk j (buffer b): wait for its count, re-run on overflow, copy its results out
  auto drain = [&](int b, int64_t off, int64_t m) -> int {
    cudaError_t e2 = cudaEventSynchronize(probed[b]);
    if (e2 != cudaSuccess) return check_cuda(e2, fn);
    int64_t cnt = (int64_t)h_tot[b];
    if (cnt > cap_b[b]) {                       // 2-pass Map for this chunk
      e2 = cudaStreamSynchronize(ds);
      if (e2 == cudaSuccess) e2 = cudaStreamSynchronize(ks);
      if (e2 != cudaSuccess) return check_cuda(e2, fn);
      cudaFreeAsync(d_ids[b], ks); d_ids[b] = nullptr;
      if (d_polys[b]) cudaFreeAsync(d_polys[b], ks);
      d_polys[b] = nullptr;
      e2 = cudaMallocAsync((void**)&d_ids[b], cnt * 8, ks);
      if (e2 == cudaSuccess && pairs) e2 = cudaMallocAsync((void**)&d_polys[b], cnt * 4, ks);
      if (e2 != cudaSuccess) return check_cuda(e2, fn);
      cap_b[b] = cnt;
      int rc = probe(b, off, m);
      if (rc != SPADE_OK) return rc;
      e2 = cudaEventSynchronize(probed[b]);
      if (e2 != cudaSuccess) return check_cuda(e2, fn);
      cnt = (int64_t)h_tot[b];
    }
    const int64_t keep = std::max<int64_t>(0, std::min(cnt, capacity - total));
    e2 = cudaStreamWaitEvent(ds, probed[b], 0);
    if (e2 == cudaSuccess && keep > 0)
      e2 = cudaMemcpyAsync(out_ids + total, d_ids[b], keep * 8, cudaMemcpyDeviceToHost, ds);
    if (e2 == cudaSuccess && keep > 0 && pairs)
      e2 = cudaMemcpyAsync(out_polys + total, d_polys[b], keep * 4, cudaMemcpyDeviceToHost, ds);
    if (e2 == cudaSuccess) e2 = cudaEventRecord(drained[b], ds);
    total += cnt;
    return check_cuda(e2, fn);
  };
  int64_t prev_off = -1, prev_m = 0;
  int64_t k = 0;
  for (int64_t off = 0; off < n; off += chunk, ++k) {
    const int b = (int)(k & 1);
    const int64_t m = std::min(chunk, n - off);
    if (k >= 2) {
      MTRY(cudaStreamWaitEvent(cs, consumed[b], 0), "wait");   // staging b free (probe k-2 done)
      MTRY(cudaStreamWaitEvent(ks, drained[b], 0), "wait");    // results b copied out (chunk k-2)
    }
    MTRY(cudaMemcpyAsync(stage[b], xy_host + 2 * off, m * 8, cudaMemcpyHostToDevice, cs), "H2D");
    MTRY(cudaEventRecord(copied[b], cs), "event");
    MTRY(cudaStreamWaitEvent(ks, copied[b], 0), "wait");
    MRC(probe(b, off, m));
    MTRY(cudaEventRecord(consumed[b], ks), "event");
    if (prev_off >= 0) MRC(drain(b ^ 1, prev_off, prev_m));
    prev_off = off;
    prev_m = m;
  }
  if (prev_off >= 0) MRC(drain((int)((k - 1) & 1), prev_off, prev_m));
  MTRY(cudaStreamSynchronize(ds), "sync");
  MTRY(cudaStreamSynchronize(ks), "sync");
  MTRY(cudaEventRecord(consumed[0], ks), "event");   // make the caller's stream observe completion
  MTRY(cudaStreamWaitEvent(st, consumed[0], 0), "wait");
  cleanup();
  *n_out = total;
  if (total > capacity)
    return set_error(SPADE_ERR_CAPACITY, "%s: %lld results exceed capacity %lld", fn, (long long)total,
                     (long long)capacity);
  return SPADE_OK;
#undef MRC
#undef MTRY
}

int spade_select_host(const spade_canvas* c, const int32_t* xy_host, int64_t n, int64_t point_id_base,
                      int64_t* out_ids_host, int64_t capacity, int64_t* n_out, spade_stream_t stream) {
  int rc = check_points(c, xy_host, n, "spade_select_host");
  if (rc) return rc;
  if (!n_out) return set_error(SPADE_ERR_INVALID_ARG, "spade_select_host: n_out is NULL");
  if (capacity < 0) return set_error(SPADE_ERR_INVALID_ARG, "spade_select_host: negative capacity");
  if (capacity > 0 && !out_ids_host) return set_error(SPADE_ERR_INVALID_ARG, "spade_select_host: out_ids_host is NULL");
  *n_out = 0;
  if (n == 0) return SPADE_OK;
  return map_host(c, xy_host, n, point_id_base, out_ids_host, nullptr, capacity, n_out, (cudaStream_t)stream,
                  "spade_select_host");
}

int spade_join_pairs_host(const spade_canvas* c, const int32_t* xy_host, int64_t n, int64_t point_id_base,
                          int64_t* out_point_ids_host, int32_t* out_poly_ids_host, int64_t capacity, int64_t* n_out,
                          spade_stream_t stream) {
  int rc = check_points(c, xy_host, n, "spade_join_pairs_host");
  if (rc) return rc;
  if (!n_out) return set_error(SPADE_ERR_INVALID_ARG, "spade_join_pairs_host: n_out is NULL");
  if (capacity < 0) return set_error(SPADE_ERR_INVALID_ARG, "spade_join_pairs_host: negative capacity");
  if (capacity > 0 && (!out_point_ids_host || !out_poly_ids_host))
    return set_error(SPADE_ERR_INVALID_ARG, "spade_join_pairs_host: output arrays are NULL");
  *n_out = 0;
  if (n == 0) return SPADE_OK;
  return map_host(c, xy_host, n, point_id_base, out_point_ids_host, out_poly_ids_host, capacity, n_out,
                  (cudaStream_t)stream, "spade_join_pairs_host");
}

// ---- kNN (knn.cu) -----------------------------------------------------------------------------
static bool knn_q_ok(int32_t qx, int32_t qy) {
  return qx >= -(1 << 30) && qx < (1 << 30) && qy >= -(1 << 30) && qy < (1 << 30);
}

int spade_knn_histogram(const int32_t* xy, int64_t n, int32_t qx, int32_t qy, int64_t* hist, spade_stream_t stream) {
  if (n < 0 || (n > 0 && (!xy || !hist))) return set_error(SPADE_ERR_INVALID_ARG, "spade_knn_histogram: bad arguments");
  if (n > 0 && ((uintptr_t)xy & 7)) return set_error(SPADE_ERR_INVALID_ARG, "spade_knn_histogram: xy must be 8-byte aligned");
  if (!knn_q_ok(qx, qy)) return set_error(SPADE_ERR_COORD_RANGE, "spade_knn_histogram: query outside [-2^30, 2^30)");
  return knn_hist(xy, n, qx, qy, hist, (cudaStream_t)stream);
}

int spade_knn_radius(const int64_t* hist_host, int64_t k, int64_t* r2_out, int64_t* count_out) {
  if (!hist_host || !r2_out || !count_out || k < 0) return set_error(SPADE_ERR_INVALID_ARG, "spade_knn_radius: bad arguments");
  int64_t acc = 0;
  for (int b = 0; b < kKnnBins; ++b) {
    acc += hist_host[b];
    if (acc >= k || b == kKnnBins - 1) {
      *r2_out = (int64_t)knn_bucket_r2(b);
      *count_out = acc;
      return SPADE_OK;
    }
  }
  return SPADE_OK;
}

int spade_knn_select(const int32_t* xy, int64_t n, int64_t point_id_base, int32_t qx, int32_t qy, int64_t r2,
                     int64_t* out_ids, int64_t* out_d2, int64_t capacity, int64_t* n_out, spade_stream_t stream) {
  if (n < 0 || (n > 0 && !xy) || (capacity > 0 && (!out_ids || !out_d2)) || r2 < 0 || point_id_base < 0)
    return set_error(SPADE_ERR_INVALID_ARG, "spade_knn_select: bad arguments");
  if (n > 0 && ((uintptr_t)xy & 7)) return set_error(SPADE_ERR_INVALID_ARG, "spade_knn_select: xy must be 8-byte aligned");
  if (!knn_q_ok(qx, qy)) return set_error(SPADE_ERR_COORD_RANGE, "spade_knn_select: query outside [-2^30, 2^30)");
  return run_with_capacity(capacity, n_out, (cudaStream_t)stream, "spade_knn_select", [&](unsigned long long* t) {
    return knn_select(xy, n, point_id_base, qx, qy, (uint64_t)r2, out_ids, out_d2, capacity, t, (cudaStream_t)stream);
  });
}

int spade_knn_topk(const int64_t* ids, const int64_t* d2, int64_t m, int64_t k, int64_t* out_ids, int64_t* out_d2,
                   spade_stream_t stream) {
  if (m < 0 || k < 0 || (m > 0 && k > 0 && (!ids || !d2 || !out_ids)))
    return set_error(SPADE_ERR_INVALID_ARG, "spade_knn_topk: bad arguments");
  return knn_topk(ids, d2, m, k, out_ids, out_d2, (cudaStream_t)stream);
}

int spade_knn(const int32_t* xy, int64_t n, int64_t point_id_base, int32_t qx, int32_t qy, int64_t k, int64_t* out_ids,
              int64_t* out_d2, int64_t* n_out, spade_stream_t stream) {
  if (!n_out || k < 0 || n < 0 || (n > 0 && k > 0 && (!xy || !out_ids)) || point_id_base < 0)
    return set_error(SPADE_ERR_INVALID_ARG, "spade_knn: bad arguments");
  *n_out = 0;
  if (!knn_q_ok(qx, qy)) return set_error(SPADE_ERR_COORD_RANGE, "spade_knn: query outside [-2^30, 2^30)");
  if (n == 0 || k == 0) return SPADE_OK;
  cudaStream_t st = (cudaStream_t)stream;
  int64_t* hist = nullptr;
  cudaError_t e = cudaMallocAsync((void**)&hist, sizeof(int64_t) * (kKnnBins + 1), st);
  if (e != cudaSuccess) return check_cuda(e, "spade_knn");
  int rc = check_cuda(cudaMemsetAsync(hist, 0, sizeof(int64_t) * (kKnnBins + 1), st), "spade_knn");
  if (rc == SPADE_OK) rc = spade_knn_histogram(xy, n, qx, qy, hist, stream);
  std::vector<int64_t> h(kKnnBins + 1, 0);
  if (rc == SPADE_OK) {
    rc = check_cuda(cudaMemcpyAsync(h.data(), hist, sizeof(int64_t) * (kKnnBins + 1), cudaMemcpyDeviceToHost, st), "spade_knn");
    if (rc == SPADE_OK) rc = check_cuda(cudaStreamSynchronize(st), "spade_knn");
  }
  cudaFreeAsync(hist, st);
  if (rc != SPADE_OK) return rc;
  if (h[kKnnBins] > 0)
    return set_error(SPADE_ERR_COORD_RANGE, "spade_knn: %lld points outside [-2^30, 2^30)", (long long)h[kKnnBins]);
  int64_t r2 = 0, m = 0;
  spade_knn_radius(h.data(), k, &r2, &m);
  if (m == 0) return SPADE_OK;
  int64_t* cand = nullptr;
  e = cudaMallocAsync((void**)&cand, sizeof(int64_t) * 2 * (size_t)m, st);
  if (e != cudaSuccess) return check_cuda(e, "spade_knn candidates");
  int64_t got = 0;
  rc = spade_knn_select(xy, n, point_id_base, qx, qy, r2, cand, cand + m, m, &got, stream);
  if (rc == SPADE_OK && got != m) rc = set_error(SPADE_ERR_INTERNAL, "spade_knn: %lld candidates, expected %lld", (long long)got, (long long)m);
  if (rc == SPADE_OK) rc = spade_knn_topk(cand, cand + m, m, k, out_ids, out_d2, stream);
  if (rc == SPADE_OK) rc = check_cuda(cudaStreamSynchronize(st), "spade_knn");
  cudaFreeAsync(cand, st);
  if (rc == SPADE_OK) *n_out = std::min(k, m);
  return rc;
}

int64_t spade_launch_count(void) { return g_launches.load(); }

int spade_last_call_stages(float* ms, int32_t cap) {
  if (cap < 0 || (cap > 0 && !ms)) return set_error(SPADE_ERR_INVALID_ARG, "spade_last_call_stages: bad arguments");
  return spade::last_call_stages(ms, cap);
}


int spade_set_option(const char* name, int64_t value) {
  using spade::set_error;
  if (!name) return set_error(SPADE_ERR_INVALID_ARG, "spade_set_option: name is NULL");
  spade::Options& o = spade::options();
  const std::string n(name);
  const bool bit = value == 0 || value == 1;
  if (n == "defer" && bit) o.defer = (int)value;
  else if (n == "count_global" && bit) o.count_global = (int)value;
  else if (n == "global_queue" && bit) o.global_queue = (int)value;
  else if (n == "debug_defer" && bit) o.debug_defer = (int)value;
  else if (n == "defer_xy" && bit) o.defer_xy = (int)value;
  else if (n == "l2_frac_pct" && value >= 1 && value <= 100) o.l2_frac_pct = (int)value;
  else if (n == "multi_agg" && bit) o.multi_agg = (int)value;
  else if (n == "k_agg" && (value == -1 || bit)) o.k_agg = (int)value;
  else if (n == "cache_slots" && (value == 0 || (value >= 1024 && value <= (1 << 16) && (value & (value - 1)) == 0)))
    o.cache_slots = (int)value;
  else if (n == "pipe" && (value == -1 || bit)) o.pipe = (int)value;
  else if (n == "host_chunk" && value >= 256 && value <= ((int64_t)1 << 28)) o.host_chunk = value;
  else if (n == "max_launch_points" && value >= 256 && value <= (1ll << 31) - 64) o.max_launch_points = value;
  else if (n == "defer_budget_mb" && value >= 64 && value <= (1ll << 20)) o.defer_budget_mb = value;
  else if (n == "fine16" && bit) o.fine16 = (int)value;
  else if (n == "stage_events" && bit) o.stage_events = (int)value;
  else if (n == "tma" && bit) o.tma = (int)value;
  else if (n == "smem_pad_kb" && value >= 0 && value <= 64) o.smem_pad_kb = (int)value;
  else if (n == "tma_slack_kb" && value >= 0 && value <= 31) o.tma_slack_kb = (int)value;
  else if (n == "pipe_notile" && bit) o.pipe_notile = (int)value;
  else if (n == "hist_copies_max" && value >= 1 && value <= 32 && (value & (value - 1)) == 0) o.hist_copies_max = (int)value;
  else if (n == "idx_queue" && (value == -1 || bit)) o.idx_queue = (int)value;
  else if (n == "coop" && (value == -1 || value == 0 || value == 4 || value == 8 || value == 16)) o.coop = (int)value;
  else return set_error(SPADE_ERR_INVALID_ARG, "spade_set_option: bad option %s = %lld", name, (long long)value);
  return SPADE_OK;
}

const char* spade_status_string(int code) {
  switch (code) {
    case SPADE_OK: return "ok";
    case SPADE_ERR_INVALID_ARG: return "invalid argument";
    case SPADE_ERR_COORD_RANGE: return "polygon coordinate outside [-2^30, 2^30)";
    case SPADE_ERR_CAPACITY: return "output capacity too small";
    case SPADE_ERR_CUDA: return "CUDA error";
    case SPADE_ERR_OOM: return "out of memory";
    case SPADE_ERR_INTERNAL: return "internal error";
    default: return "unknown status";
  }
}

const char* spade_last_error(void) { return g_err; }

}  // extern "C"
