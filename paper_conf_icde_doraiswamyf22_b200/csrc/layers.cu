// layers.cu — the paper's layer index for overlapping polygon sets.
//
// The paper draws polygons into a texture whose pixels hold ONE polygon each, so a set whose
// polygons overlap is split into layers of mutually non-intersecting polygons, one canvas (and one
// selection pass over the points) per layer; the layers are built iteratively by blend / mask
// passes.  Here the canvas itself is exact for overlaps (owner sets), so
// the layer index is the alternative plan this file provides for comparison (SURVEY.md §8(f)
// NEXT(4), "layer index ... vs multi-owner pixels"):
//   * conflicts = the closed-intersection pairs of the set with itself (spade_join_polygons: the
//     polygon x polygon join of P:202; touching polygons conflict too, which is conservative);
//   * layers = a greedy colouring of the conflict graph (Welsh-Powell: by decreasing degree, each
//     polygon takes the smallest layer none of its conflicting polygons holds), on the host;
//   * one canvas per layer over ALL P polygon slots, the other layers' polygons given no rings, so
//     every layer's COUNT accumulates into the same global counts with global polygon ids;
//   * COUNT = one probe pass per layer (spade_join_count, which accumulates).
#include <algorithm>
#include <numeric>
#include <vector>
#include "spade_internal.cuh"

struct spade_layered {
  int device = 0;
  int32_t P = 0, L = 0;
  std::vector<spade_canvas*> cv;        // one canvas per layer (P slots each)
  std::vector<int32_t> layer_of;        // [P] layer of every polygon
  std::vector<float> build_ms;          // per-layer build time of the last build (host wall clock)
};

extern "C" {

int spade_layer_assign(const int32_t* pair_a, const int32_t* pair_b, int64_t npairs, int32_t P, int32_t* layer_of,
                       int32_t* num_layers) {
  using spade::set_error;
  if (P < 0 || npairs < 0 || (npairs > 0 && (!pair_a || !pair_b)) || (P > 0 && !layer_of) || !num_layers)
    return set_error(SPADE_ERR_INVALID_ARG, "spade_layer_assign: bad arguments");
  std::vector<int64_t> deg(P + 1, 0);
  for (int64_t i = 0; i < npairs; ++i) {
    const int32_t a = pair_a[i], b = pair_b[i];
    if (a < 0 || a >= P || b < 0 || b >= P) return set_error(SPADE_ERR_INVALID_ARG, "spade_layer_assign: polygon id out of range");
    if (a != b) { ++deg[a]; ++deg[b]; }
  }
  // adjacency in CSR (both directions; duplicates harmless)
  std::vector<int64_t> off(P + 1, 0);
  for (int32_t p = 0; p < P; ++p) off[p + 1] = off[p] + deg[p];
  std::vector<int32_t> adj(off[P]);
  std::vector<int64_t> fill(off.begin(), off.end() - 1);
  for (int64_t i = 0; i < npairs; ++i) {
    const int32_t a = pair_a[i], b = pair_b[i];
    if (a != b) { adj[fill[a]++] = b; adj[fill[b]++] = a; }
  }
  std::vector<int32_t> order(P);
  std::iota(order.begin(), order.end(), 0);
  std::stable_sort(order.begin(), order.end(), [&](int32_t x, int32_t y) { return deg[x] > deg[y]; });
  std::fill(layer_of, layer_of + P, -1);
  std::vector<int32_t> mark;                          // mark[l] == p: layer l is taken by a neighbour of p
  int32_t L = 0;
  for (int32_t p : order) {
    for (int64_t j = off[p]; j < off[p + 1]; ++j) {
      const int32_t l = layer_of[adj[j]];
      if (l >= 0) mark[l] = p;
    }
    int32_t l = 0;
    while (l < L && mark[l] == p) ++l;
    if (l == L) { mark.push_back(-1); ++L; }
    layer_of[p] = l;
  }
  *num_layers = L;
  return SPADE_OK;
}

int spade_build_layered(const int32_t* ring_xy, const int64_t* ring_off, const int64_t* poly_ring_off, int32_t P,
                        const spade_canvas_params* prm, spade_stream_t stream, spade_layered** out) {
  using spade::set_error;
  using spade::check_cuda;
  if (!out) return set_error(SPADE_ERR_INVALID_ARG, "spade_build_layered: out is NULL");
  *out = nullptr;
  if (P < 0 || (P > 0 && (!ring_xy || !ring_off || !poly_ring_off)))
    return set_error(SPADE_ERR_INVALID_ARG, "spade_build_layered: bad arguments");
  cudaStream_t st = (cudaStream_t)stream;
  auto* lc = new spade_layered;
  cudaGetDevice(&lc->device);
  lc->P = P;
  lc->layer_of.assign(P, 0);
  auto fail = [&](int rc) { spade_layered_free(lc); return rc; };
  // 1. conflicts: the closed-intersection self-join (capacity protocol: one retry)
  int64_t cap = std::max<int64_t>(4 * (int64_t)P, 1024), npairs = 0;
  int32_t *da = nullptr, *db = nullptr;
  for (int attempt = 0; attempt < 2; ++attempt) {
    cudaError_t e = cudaMallocAsync((void**)&da, sizeof(int32_t) * cap, st);
    if (e == cudaSuccess) e = cudaMallocAsync((void**)&db, sizeof(int32_t) * cap, st);
    if (e != cudaSuccess) return fail(check_cuda(e, "spade_build_layered: pairs"));
    const int rc = P > 0 ? spade_join_polygons(ring_xy, ring_off, poly_ring_off, P, ring_xy, ring_off, poly_ring_off, P, prm,
                                               da, db, cap, &npairs, stream)
                         : SPADE_OK;
    if (rc == SPADE_ERR_CAPACITY && attempt == 0) {
      cudaFreeAsync(da, st); cudaFreeAsync(db, st); da = db = nullptr;
      cap = npairs;
      continue;
    }
    if (rc != SPADE_OK) { cudaFreeAsync(da, st); cudaFreeAsync(db, st); return fail(rc); }
    break;
  }
  std::vector<int32_t> ha(npairs), hb(npairs);
  if (npairs > 0) {
    cudaMemcpyAsync(ha.data(), da, sizeof(int32_t) * npairs, cudaMemcpyDeviceToHost, st);
    cudaMemcpyAsync(hb.data(), db, sizeof(int32_t) * npairs, cudaMemcpyDeviceToHost, st);
  }
  cudaFreeAsync(da, st); cudaFreeAsync(db, st);
  // 2. the polygon arrays on the host (ring structure; vertices gathered per layer below)
  std::vector<int64_t> hpro(P + 1);
  cudaError_t e = P > 0 ? cudaMemcpyAsync(hpro.data(), poly_ring_off, sizeof(int64_t) * (P + 1), cudaMemcpyDeviceToHost, st) : cudaSuccess;
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return fail(check_cuda(e, "spade_build_layered: copy"));
  const int64_t R = P > 0 ? hpro[P] : 0;
  std::vector<int64_t> hro(R + 1, 0);
  if (P > 0) e = cudaMemcpyAsync(hro.data(), ring_off, sizeof(int64_t) * (R + 1), cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return fail(check_cuda(e, "spade_build_layered: copy"));
  const int64_t V = hro[R];
  std::vector<int32_t> hxy(2 * V);
  if (V > 0) e = cudaMemcpyAsync(hxy.data(), ring_xy, sizeof(int32_t) * 2 * V, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return fail(check_cuda(e, "spade_build_layered: copy"));
  // 3. layers
  int32_t L = 0;
  int rc = spade_layer_assign(ha.data(), hb.data(), npairs, P, lc->layer_of.data(), &L);
  if (rc != SPADE_OK) return fail(rc);
  lc->L = L;
  // 4. one canvas per layer, P polygon slots (the other layers' polygons without rings)
  for (int32_t l = 0; l < L; ++l) {
    std::vector<int32_t> xy;
    std::vector<int64_t> ro(1, 0), pro(P + 1, 0);
    for (int32_t p = 0; p < P; ++p) {
      if (lc->layer_of[p] == l)
        for (int64_t r = hpro[p]; r < hpro[p + 1]; ++r) {
          xy.insert(xy.end(), hxy.begin() + 2 * hro[r], hxy.begin() + 2 * hro[r + 1]);
          ro.push_back((int64_t)xy.size() / 2);
        }
      pro[p + 1] = (int64_t)ro.size() - 1;
    }
    int32_t* dxy = nullptr;
    int64_t *dro = nullptr, *dpro = nullptr;
    e = cudaMallocAsync((void**)&dxy, sizeof(int32_t) * std::max<size_t>(xy.size(), 2), st);
    if (e == cudaSuccess) e = cudaMallocAsync((void**)&dro, sizeof(int64_t) * ro.size(), st);
    if (e == cudaSuccess) e = cudaMallocAsync((void**)&dpro, sizeof(int64_t) * pro.size(), st);
    if (e == cudaSuccess && !xy.empty()) e = cudaMemcpyAsync(dxy, xy.data(), sizeof(int32_t) * xy.size(), cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) e = cudaMemcpyAsync(dro, ro.data(), sizeof(int64_t) * ro.size(), cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) e = cudaMemcpyAsync(dpro, pro.data(), sizeof(int64_t) * pro.size(), cudaMemcpyHostToDevice, st);
    spade_canvas* cv = nullptr;
    rc = e == cudaSuccess ? spade_build_canvas(dxy, dro, dpro, P, prm, stream, &cv) : check_cuda(e, "spade_build_layered: layer arrays");
    cudaStreamSynchronize(st);                        // (the host vectors die at the end of this iteration)
    cudaFreeAsync(dxy, st); cudaFreeAsync(dro, st); cudaFreeAsync(dpro, st);
    if (rc != SPADE_OK) return fail(rc);
    lc->cv.push_back(cv);
  }
  *out = lc;
  return SPADE_OK;
}

int spade_join_count_layered(const spade_layered* lc, const int32_t* xy, int64_t n, int64_t* counts, spade_stream_t stream) {
  using spade::set_error;
  if (!lc) return set_error(SPADE_ERR_INVALID_ARG, "spade_join_count_layered: layered canvas is NULL");
  for (spade_canvas* cv : lc->cv) {                  // one probe pass per layer, accumulating
    const int rc = spade_join_count(cv, xy, n, counts, stream);
    if (rc != SPADE_OK) return rc;
  }
  return SPADE_OK;
}

int spade_layered_info(const spade_layered* lc, int32_t* num_layers, int32_t* layer_of) {
  using spade::set_error;
  if (!lc || !num_layers) return set_error(SPADE_ERR_INVALID_ARG, "spade_layered_info: bad arguments");
  *num_layers = lc->L;
  if (layer_of) std::copy(lc->layer_of.begin(), lc->layer_of.end(), layer_of);
  return SPADE_OK;
}

void spade_layered_free(spade_layered* lc) {
  if (!lc) return;
  for (spade_canvas* cv : lc->cv) spade_canvas_free(cv);
  delete lc;
}

}  // extern "C"
