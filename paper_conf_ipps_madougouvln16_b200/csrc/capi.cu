// capi.cu -- the C ABI of include/bf.h: argument checks, error codes,
// allocator hook, host/device pointer staging, forest import/export, and the
// single-step parity entry points.
#include <cstdio>
#include <cstring>
#include <atomic>
#include <mutex>

#include "bf_internal.cuh"

namespace bf {

static thread_local std::string g_last_error;
void set_error(const std::string& m) { g_last_error = m; }

static bf_alloc_fn g_alloc = nullptr;
static bf_free_fn g_free = nullptr;
static void* g_ctx = nullptr;
static std::atomic<int64_t> g_budget{0};
int64_t memory_budget() { return g_budget.load(); }

void* dev_alloc(size_t bytes, cudaStream_t s) {
  if (bytes == 0) return nullptr;
  void* p = nullptr;
  if (g_alloc) {
    p = g_alloc(bytes, (void*)s, g_ctx);
    BF_REQUIRE(p != nullptr, BF_ENOMEM, "allocator hook returned NULL for " + std::to_string(bytes) + " bytes");
    return p;
  }
  static bool pool_cfg = false;
  if (!pool_cfg) {
    // keep freed blocks cached in the device pool (no unmap/remap of the GBs of
    // per-fit work space at every synchronisation point)
    int dev = 0;
    cudaGetDevice(&dev);
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
      uint64_t thr = UINT64_MAX;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    pool_cfg = true;
  }
  cudaError_t e = cudaMallocAsync(&p, bytes, s);
  if (e != cudaSuccess) {
    cudaGetLastError();
    throw Error{BF_ENOMEM, "cudaMallocAsync(" + std::to_string(bytes) + ") failed: " + cudaGetErrorString(e)};
  }
  return p;
}

void dev_free(void* p, cudaStream_t s) {
  if (!p) return;
  if (g_free) {
    g_free(p, (void*)s, g_ctx);
    return;
  }
  cudaFreeAsync(p, s);
}

bool is_device_ptr(const void* p) {
  if (!p) return true;
  cudaPointerAttributes a;
  cudaError_t e = cudaPointerGetAttributes(&a, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

InStage::InStage(const void* ptr, size_t bytes, cudaStream_t s) {
  if (is_device_ptr(ptr)) {
    dptr = ptr;
    return;
  }
  tmp.alloc(bytes, s);
  BF_CUDA_CHECK(cudaMemcpyAsync(tmp.p, ptr, bytes, cudaMemcpyHostToDevice, s));
  dptr = tmp.p;
}

OutStage::OutStage(void* ptr, size_t b, cudaStream_t s) : bytes(b) {
  if (is_device_ptr(ptr)) {
    dptr = ptr;
    return;
  }
  host = ptr;
  tmp.alloc(b, s);
  dptr = tmp.p;
}

void OutStage::finish(cudaStream_t s) {
  if (host && bytes) BF_CUDA_CHECK(cudaMemcpyAsync(host, dptr, bytes, cudaMemcpyDeviceToHost, s));
}

void forest_alloc(bf_forest* f, int64_t total, int32_t ntrees, cudaStream_t s) {
  f->stream = s;
  f->info.total_nodes = total;
  size_t t = (size_t)(total > 0 ? total : 1);
  f->d_nodes = (Node16*)dev_alloc(t * sizeof(Node16), s);
  f->d_count = (int32_t*)dev_alloc(t * sizeof(int32_t), s);
  f->d_value = (double*)dev_alloc(t * sizeof(double), s);
  f->d_drss = (double*)dev_alloc(t * sizeof(double), s);
  f->d_tree_off = (int64_t*)dev_alloc((size_t)(ntrees + 1) * sizeof(int64_t), s);
}

void forest_release(bf_forest* f) {
  // Freed stream-ordered on the allocation stream.  If a call (predict, importance, ...) used the forest on
  // another stream, its kernels may still read the arrays: wait for the device first, so neither
  // cudaFreeAsync nor a caching allocator (torch) can hand the blocks out while they are in use.
  if (f->foreign_stream) cudaDeviceSynchronize();
  cudaStream_t s = f->stream;
  dev_free(f->d_nodes, s);
  dev_free(f->d_count, s);
  dev_free(f->d_value, s);
  dev_free(f->d_drss, s);
  dev_free(f->d_tree_off, s);
  if (f->d_nodes8) dev_free(f->d_nodes8, s);
  if (f->d_roots8) dev_free(f->d_roots8, s);
  f->d_nodes8 = nullptr;
  f->d_roots8 = nullptr;
  f->nodes8_state = 0;
  if (f->d_g32) dev_free(f->d_g32, s);
  if (f->d_g32_root) dev_free(f->d_g32_root, s);
  f->d_g32 = nullptr;
  f->d_g32_root = nullptr;
  f->g32_state = 0;
  f->d_nodes = nullptr;
}

__global__ void k_philox(const uint32_t* ctr, uint32_t k0, uint32_t k1, uint32_t* out, int64_t count) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= count) return;
  uint32_t x[4];
  philox4x32_10(ctr[4 * i], ctr[4 * i + 1], ctr[4 * i + 2], ctr[4 * i + 3], k0, k1, x);
  for (int j = 0; j < 4; ++j) out[4 * i + j] = x[j];
}

void philox_impl(const uint32_t* ctr, uint32_t k0, uint32_t k1, uint32_t* out, int64_t count, cudaStream_t s) {
  if (count <= 0) return;
  k_philox<<<(unsigned)ceil_div(count, 256), 256, 0, s>>>(ctr, k0, k1, out, count);
  BF_CUDA_CHECK(cudaGetLastError());
}

__global__ void k_i128(const int64_t* hi, const uint64_t* lo, double* out, int64_t count) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= count) return;
  __int128 v = (__int128)(((unsigned __int128)(uint64_t)hi[i] << 64) | (unsigned __int128)lo[i]);
  out[i] = i128_to_double(v);
}

void i128_impl(const int64_t* hi, const uint64_t* lo, double* out, int64_t count, cudaStream_t s) {
  if (count <= 0) return;
  k_i128<<<(unsigned)ceil_div(count, 256), 256, 0, s>>>(hi, lo, out, count);
  BF_CUDA_CHECK(cudaGetLastError());
}

}  // namespace bf

using namespace bf;

#define BF_API_BEGIN try {
#define BF_API_END                                   \
  }                                                  \
  catch (const bf::Error& e) {                       \
    bf::set_error(e.msg);                            \
    return e.code;                                   \
  }                                                  \
  catch (const std::exception& e) {                  \
    bf::set_error(std::string("exception: ") + e.what()); \
    return BF_ECUDA;                                 \
  }                                                  \
  return BF_OK;

extern "C" {

const char* bf_version(void) { return "blackforest-b200 1 (sm_100a)"; }
const char* bf_last_error(void) { return g_last_error.c_str(); }

int bf_set_allocator(bf_alloc_fn alloc, bf_free_fn free_, void* ctx) {
  g_alloc = alloc;
  g_free = free_;
  g_ctx = ctx;
  return BF_OK;
}

int bf_set_memory_budget(int64_t bytes) {
  if (bytes < 0) return BF_EINVAL;
  bf::g_budget.store(bytes);
  return BF_OK;
}

int bf_release_workspace(void) {
  BF_API_BEGIN
  BF_REQUIRE(bf::release_list_workspace(), BF_EINVAL, "bf_release_workspace: a fit is using the work space");
  BF_API_END
}

int bf_fit(const double* X, int64_t ldx, const double* y, int64_t n, int32_t p, const bf_params* prm, void* stream,
           bf_forest** out) {
  BF_API_BEGIN
  BF_REQUIRE(out && prm && X && y, BF_EINVAL, "bf_fit: NULL argument");
  *out = nullptr;
  BF_REQUIRE(n >= 1 && p >= 1 && ldx >= n, BF_EINVAL, "bf_fit: need n >= 1, p >= 1, ldx >= n");
  BF_REQUIRE(n < (int64_t(1) << 31), BF_ERANGE, "bf_fit: n >= 2^31");
  fit_impl(X, ldx, y, n, p, *prm, (cudaStream_t)stream, out);
  BF_API_END
}

void bf_forest_free(bf_forest* f) {
  if (!f) return;
  forest_release(f);
  delete f;
}

int bf_forest_info_get(const bf_forest* f, bf_forest_info* info) {
  if (!f || !info) {
    set_error("bf_forest_info_get: NULL");
    return BF_EINVAL;
  }
  *info = f->info;
  return BF_OK;
}

__global__ void k_unpack_nodes(const Node16* nodes, int64_t total, int32_t* feature, int32_t* left, double* tv) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= total) return;
  Node16 nd = nodes[i];
  feature[i] = nd.feature;
  left[i] = nd.left;
  tv[i] = nd.v;
}

int bf_forest_export(const bf_forest* f, bf_forest_view* v) {
  BF_API_BEGIN
  BF_REQUIRE(f && v, BF_EINVAL, "bf_forest_export: NULL");
  v->info = f->info;
  const int32_t nt = f->info.tree_end - f->info.tree_begin;
  const int64_t tot = f->info.total_nodes;
  cudaStream_t s = nullptr;
  if (v->tree_off) memcpy(v->tree_off, f->tree_off.data(), sizeof(int64_t) * (size_t)(nt + 1));
  if (tot > 0) {
    DBuf<int32_t> fe(tot, s), le(tot, s);
    DBuf<double> tv(tot, s);
    k_unpack_nodes<<<(unsigned)ceil_div(tot, 256), 256, 0, s>>>(f->d_nodes, tot, fe.p, le.p, tv.p);
    BF_CUDA_CHECK(cudaGetLastError());
    if (v->feature) BF_CUDA_CHECK(cudaMemcpyAsync(v->feature, fe.p, tot * 4, cudaMemcpyDeviceToHost, s));
    if (v->left) BF_CUDA_CHECK(cudaMemcpyAsync(v->left, le.p, tot * 4, cudaMemcpyDeviceToHost, s));
    if (v->thr_or_value) BF_CUDA_CHECK(cudaMemcpyAsync(v->thr_or_value, tv.p, tot * 8, cudaMemcpyDeviceToHost, s));
    if (v->count) BF_CUDA_CHECK(cudaMemcpyAsync(v->count, f->d_count, tot * 4, cudaMemcpyDeviceToHost, s));
    if (v->value) BF_CUDA_CHECK(cudaMemcpyAsync(v->value, f->d_value, tot * 8, cudaMemcpyDeviceToHost, s));
    if (v->drss) BF_CUDA_CHECK(cudaMemcpyAsync(v->drss, f->d_drss, tot * 8, cudaMemcpyDeviceToHost, s));
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
  }
  BF_API_END
}

__global__ void k_pack_nodes(Node16* nodes, int64_t total, const int32_t* feature, const int32_t* left,
                             const double* tv) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= total) return;
  Node16 nd;
  nd.feature = feature[i];
  nd.left = left[i];
  nd.v = tv[i];
  nodes[i] = nd;
}

int bf_forest_import(const bf_forest_view* v, void* stream, bf_forest** out) {
  bf_forest* f = nullptr;
  BF_API_BEGIN
  BF_REQUIRE(v && out && v->tree_off && v->feature && v->left && v->thr_or_value, BF_EINVAL,
             "bf_forest_import: NULL");
  cudaStream_t s = (cudaStream_t)stream;
  *out = nullptr;
  const int32_t nt = v->info.tree_end - v->info.tree_begin;
  BF_REQUIRE(nt >= 0 && v->info.tree_begin >= 0 && v->info.tree_end <= v->info.ntree_total, BF_EINVAL,
             "bf_forest_import: bad tree range");
  f = new bf_forest();
  f->info = v->info;
  f->tree_off.resize((size_t)nt + 1);
  {
    InStage to(v->tree_off, sizeof(int64_t) * (nt + 1), s);
    BF_CUDA_CHECK(cudaMemcpyAsync(f->tree_off.data(), to.dptr, sizeof(int64_t) * (nt + 1), cudaMemcpyDefault, s));
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
  }
  const int64_t tot = f->tree_off[nt];
  BF_REQUIRE(tot >= 0, BF_EINVAL, "bf_forest_import: negative node count");
  forest_alloc(f, tot, nt, s);
  BF_CUDA_CHECK(cudaMemcpyAsync(f->d_tree_off, f->tree_off.data(), sizeof(int64_t) * (nt + 1),
                                cudaMemcpyHostToDevice, s));
  if (tot > 0) {
    InStage fe(v->feature, tot * 4, s), le(v->left, tot * 4, s), tv(v->thr_or_value, tot * 8, s);
    k_pack_nodes<<<(unsigned)ceil_div(tot, 256), 256, 0, s>>>(f->d_nodes, tot, (const int32_t*)fe.dptr,
                                                               (const int32_t*)le.dptr, (const double*)tv.dptr);
    BF_CUDA_CHECK(cudaGetLastError());
    if (v->count) BF_CUDA_CHECK(cudaMemcpyAsync(f->d_count, v->count, tot * 4, cudaMemcpyDefault, s));
    else BF_CUDA_CHECK(cudaMemsetAsync(f->d_count, 0, tot * 4, s));
    if (v->value) BF_CUDA_CHECK(cudaMemcpyAsync(f->d_value, v->value, tot * 8, cudaMemcpyDefault, s));
    else BF_CUDA_CHECK(cudaMemsetAsync(f->d_value, 0, tot * 8, s));
    if (v->drss) BF_CUDA_CHECK(cudaMemcpyAsync(f->d_drss, v->drss, tot * 8, cudaMemcpyDefault, s));
    else BF_CUDA_CHECK(cudaMemsetAsync(f->d_drss, 0, tot * 8, s));
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
  }
  *out = f;
  f = nullptr;
  } catch (const bf::Error& e) {
    if (f) bf_forest_free(f);
    bf::set_error(e.msg);
    return e.code;
  }
  return BF_OK;
}

int bf_predict(const bf_forest* f, const double* Xq, int64_t ldq, int64_t m, double* yhat_sum, double* yhat,
               int32_t ntree_total, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(f && (Xq || m == 0), BF_EINVAL, "bf_predict: NULL");
  BF_REQUIRE(m >= 0 && ldq >= m, BF_EINVAL, "bf_predict: need m >= 0, ldq >= m");
  f->touch((cudaStream_t)stream);
  predict_impl(f, Xq, ldq, m, yhat_sum, yhat, ntree_total, (cudaStream_t)stream);
  BF_API_END
}

int bf_pd_grid(const double* x, int64_t n, int32_t n_pt, double* grid, int32_t* G, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(x && grid && G, BF_EINVAL, "bf_pd_grid: NULL");
  BF_REQUIRE(n >= 1 && n < (int64_t(1) << 31) && n_pt >= 1, BF_EINVAL, "bf_pd_grid: need 1 <= n < 2^31, n_pt >= 1");
  pd_grid_impl(x, n, n_pt, grid, G, (cudaStream_t)stream);
  BF_API_END
}

int bf_partial_dependence(const bf_forest* f, const double* X, int64_t ldx, int64_t n, int32_t p, int32_t m,
                          const double* grid, int32_t G, double* pd_sum, double* pd, int32_t ntree_total,
                          void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(f && X && grid, BF_EINVAL, "bf_partial_dependence: NULL");
  BF_REQUIRE(p == f->info.p && n >= 0 && ldx >= n && m >= 0 && m < p && G >= 1, BF_EINVAL,
             "bf_partial_dependence: need p == forest p, ldx >= n, 0 <= m < p, G >= 1");
  f->touch((cudaStream_t)stream);
  partial_dependence_impl(f, X, ldx, n, m, grid, G, pd_sum, pd, ntree_total, (cudaStream_t)stream);
  BF_API_END
}

int bf_oob_importance(const bf_forest* f, const double* X, int64_t ldx, const double* y, int64_t n, int32_t p,
                      const bf_oob_accum* acc, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(f && X && y && acc, BF_EINVAL, "bf_oob_importance: NULL");
  BF_REQUIRE(n == f->info.n && p == f->info.p && ldx >= n, BF_EINVAL,
             "bf_oob_importance: X/y shape differs from the training data");
  f->touch((cudaStream_t)stream);
  oob_importance_impl(f, X, ldx, y, n, p, *acc, (cudaStream_t)stream);
  BF_API_END
}

int bf_importance_finalize(const double* d_slots, const double* npur_slots, const double* oob_sum,
                           const int32_t* oob_cnt, const double* y, int64_t n, int32_t p, int32_t ntree,
                           double* inc_mse, double* inc_mse_raw, double* inc_mse_sd, double* inc_node_purity,
                           double* oob_mse, double* rsq, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(d_slots && npur_slots && oob_sum && oob_cnt && y, BF_EINVAL, "bf_importance_finalize: NULL");
  BF_REQUIRE(n >= 1 && p >= 1 && ntree >= 1, BF_EINVAL, "bf_importance_finalize: bad sizes");
  cudaStream_t s = (cudaStream_t)stream;
  InStage ds(d_slots, sizeof(double) * ntree * p, s), ns(npur_slots, sizeof(double) * ntree * p, s),
      os(oob_sum, sizeof(double) * n, s), oc(oob_cnt, sizeof(int32_t) * n, s), ys(y, sizeof(double) * n, s);
  DBuf<double> o4(4 * (size_t)p, s), o2(2, s);
  importance_finalize_impl((const double*)ds.dptr, (const double*)ns.dptr, (const double*)os.dptr,
                           (const int32_t*)oc.dptr, (const double*)ys.dptr, n, p, ntree, o4.p, o2.p, s);
  double* outs[4] = {inc_mse, inc_mse_raw, inc_mse_sd, inc_node_purity};
  for (int j = 0; j < 4; ++j)
    if (outs[j]) BF_CUDA_CHECK(cudaMemcpyAsync(outs[j], o4.p + (size_t)j * p, sizeof(double) * p, cudaMemcpyDefault, s));
  if (oob_mse) BF_CUDA_CHECK(cudaMemcpyAsync(oob_mse, o2.p, sizeof(double), cudaMemcpyDefault, s));
  if (rsq) BF_CUDA_CHECK(cudaMemcpyAsync(rsq, o2.p + 1, sizeof(double), cudaMemcpyDefault, s));
  if (!is_device_ptr(inc_mse) || !is_device_ptr(oob_mse) || !is_device_ptr(rsq) || !is_device_ptr(inc_mse_raw) ||
      !is_device_ptr(inc_mse_sd) || !is_device_ptr(inc_node_purity))
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
  else
    BF_CUDA_CHECK(cudaStreamSynchronize(s));  // temporaries are freed stream-ordered; keep the call simple
  BF_API_END
}

int bf_pca(const double* X, int64_t ldx, int64_t n, int32_t p, int32_t scale, int32_t k, double* sdev,
           double* rotation, double* center, double* scores, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(X && sdev && rotation, BF_EINVAL, "bf_pca: NULL");
  BF_REQUIRE(n >= 2 && p >= 1 && ldx >= n && k >= 0 && k <= p, BF_EINVAL, "bf_pca: bad sizes");
  BF_REQUIRE(p <= 1024, BF_ENOTIMPL, "bf_pca: p > 1024");
  pca_impl(X, ldx, n, p, scale, k, sdev, rotation, center, scores, (cudaStream_t)stream);
  BF_API_END
}

int bf_pca_retained(const double* sdev, int32_t p, double frac, int32_t cap, int32_t* k, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(sdev && k, BF_EINVAL, "bf_pca_retained: NULL");
  BF_REQUIRE(p >= 1 && p <= 1024 && cap >= 1 && frac > 0.0 && frac <= 1.0, BF_EINVAL, "bf_pca_retained: bad arguments");
  pca_retained_impl(sdev, p, frac, cap, k, (cudaStream_t)stream);
  BF_API_END
}

int bf_varimax(const double* L, int64_t ldl, int32_t p, int32_t k, int32_t normalize, double eps, double* loadings,
               double* rotmat, int32_t* iters, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(L && loadings && rotmat, BF_EINVAL, "bf_varimax: NULL");
  BF_REQUIRE(p >= 1 && k >= 1 && k <= 32 && ldl >= p && eps >= 0.0, BF_EINVAL,
             "bf_varimax: need p >= 1, 1 <= k <= 32, ldl >= p, eps >= 0");
  varimax_impl(L, ldl, p, k, normalize, eps, loadings, rotmat, iters, (cudaStream_t)stream);
  BF_API_END
}

int bf_glm_gaussian(const double* Z, int64_t ldz, int64_t n, int32_t k, const double* Y, int64_t ldy, int32_t r,
                    double* coef, double* deviance, double* null_deviance, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(Z && Y && coef, BF_EINVAL, "bf_glm_gaussian: NULL");
  BF_REQUIRE(ldz >= n && ldy >= n, BF_EINVAL, "bf_glm_gaussian: need ldz >= n, ldy >= n");
  glm_gaussian_impl(Z, ldz, n, k, Y, ldy, r, coef, deviance, null_deviance, (cudaStream_t)stream);
  BF_API_END
}

int bf_glm_predict(const double* Z, int64_t ldz, int64_t n, int32_t k, const double* coef, int32_t r, double* out,
                   int64_t ldo, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(Z && coef && out, BF_EINVAL, "bf_glm_predict: NULL");
  BF_REQUIRE(ldz >= n && ldo >= n, BF_EINVAL, "bf_glm_predict: need ldz >= n, ldo >= n");
  glm_predict_impl(Z, ldz, n, k, coef, r, out, ldo, (cudaStream_t)stream);
  BF_API_END
}

int bf_mars_fit(const double* X, int64_t ldx, int64_t n, int32_t d, const double* y, int32_t nk, double thresh,
                double penalty, int32_t* nterms, int32_t* term_var, double* term_knot, int32_t* term_dir, double* coef,
                double* stats, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(X && y && nterms && term_var && term_knot && term_dir && coef && stats, BF_EINVAL, "bf_mars_fit: NULL");
  BF_REQUIRE(ldx >= n && thresh >= 0.0 && penalty >= 0.0, BF_EINVAL, "bf_mars_fit: need ldx >= n, thresh, penalty >= 0");
  mars_fit_impl(X, ldx, n, d, y, nk, thresh, penalty, nterms, term_var, term_knot, term_dir, coef, stats,
                (cudaStream_t)stream);
  BF_API_END
}

int bf_mars_predict(const double* X, int64_t ldx, int64_t m, int32_t d, int32_t nterms, const int32_t* term_var,
                    const double* term_knot, const int32_t* term_dir, const double* coef, double* out, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(X && out && (nterms == 0 || (term_var && term_knot && term_dir && coef)), BF_EINVAL, "bf_mars_predict: NULL");
  BF_REQUIRE(ldx >= m && nterms >= 0 && d >= 1, BF_EINVAL, "bf_mars_predict: need ldx >= m, d >= 1");
  for (int j = 0; j < nterms; ++j)
    BF_REQUIRE(term_var[j] >= 0 && term_var[j] < d, BF_EINVAL, "bf_mars_predict: term variable out of range");
  mars_predict_impl(X, ldx, m, d, nterms, term_var, term_knot, term_dir, coef, out, (cudaStream_t)stream);
  BF_API_END
}

int bf_rank_similarity(const double* a, const double* b, int32_t p, double* out, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(a && b && out, BF_EINVAL, "bf_rank_similarity: NULL");
  BF_REQUIRE(p >= 1, BF_EINVAL, "bf_rank_similarity: need p >= 1");
  rank_similarity_impl(a, b, p, out, (cudaStream_t)stream);
  BF_API_END
}

int bf_log_size_design(const double* size, int64_t n, double* Z, int64_t ldz, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(size && Z, BF_EINVAL, "bf_log_size_design: NULL");
  BF_REQUIRE(n >= 2 && ldz >= n, BF_EINVAL, "bf_log_size_design: need n >= 2, ldz >= n");
  log_size_design_impl(size, n, Z, ldz, (cudaStream_t)stream);
  BF_API_END
}

int bf_prediction_error(const double* yhat, const double* y, int64_t m, double* out, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(yhat && y && out, BF_EINVAL, "bf_prediction_error: NULL");
  BF_REQUIRE(m >= 1, BF_EINVAL, "bf_prediction_error: need m >= 1");
  prediction_error_impl(yhat, y, m, out, (cudaStream_t)stream);
  BF_API_END
}

int bf_philox(const uint32_t* ctr, uint32_t key0, uint32_t key1, uint32_t* out, int64_t count, void* stream) {
  BF_API_BEGIN
  cudaStream_t s = (cudaStream_t)stream;
  InStage ci(ctr, sizeof(uint32_t) * 4 * count, s);
  OutStage co(out, sizeof(uint32_t) * 4 * count, s);
  philox_impl((const uint32_t*)ci.dptr, key0, key1, (uint32_t*)co.dptr, count, s);
  co.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_API_END
}

int bf_sort_u64(uint64_t* keys, uint32_t* vals, int64_t n, int32_t nseg, void* stream) {
  BF_API_BEGIN
  cudaStream_t s = (cudaStream_t)stream;
  BF_REQUIRE(keys && n >= 0 && nseg >= 1, BF_EINVAL, "bf_sort_u64: bad arguments");
  BF_REQUIRE(is_device_ptr(keys) && is_device_ptr(vals), BF_EINVAL, "bf_sort_u64: device pointers required");
  const int64_t tot = n * nseg;
  DBuf<uint64_t> k1(tot, s);
  DBuf<uint32_t> v1(vals ? tot : 0, s);
  uint32_t* vres = nullptr;
  const uint64_t* kres = radix_sort_u64(keys, k1.p, vals, vals ? v1.p : nullptr, n, nseg, s, &vres);
  if (kres != keys && tot) BF_CUDA_CHECK(cudaMemcpyAsync(keys, kres, sizeof(uint64_t) * tot, cudaMemcpyDeviceToDevice, s));
  if (vals && vres != vals && tot) BF_CUDA_CHECK(cudaMemcpyAsync(vals, vres, sizeof(uint32_t) * tot, cudaMemcpyDeviceToDevice, s));
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_API_END
}

int bf_scan_u32(const uint32_t* in, uint32_t* out, int64_t n, int32_t inclusive, void* stream) {
  BF_API_BEGIN
  cudaStream_t s = (cudaStream_t)stream;
  BF_REQUIRE(in && out && n >= 0 && is_device_ptr(in) && is_device_ptr(out), BF_EINVAL, "bf_scan_u32: bad arguments");
  if (inclusive) scan_inclusive(in, out, n, s);
  else scan_exclusive(in, out, n, s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_API_END
}

int bf_unique_u64(const uint64_t* sorted, int64_t n, uint64_t* out, int32_t* count, void* stream) {
  BF_API_BEGIN
  cudaStream_t s = (cudaStream_t)stream;
  BF_REQUIRE(sorted && out && count && n >= 0 && is_device_ptr(sorted) && is_device_ptr(out) && is_device_ptr(count),
             BF_EINVAL, "bf_unique_u64: bad arguments");
  unique_u64(sorted, n, out, count, s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_API_END
}

int bf_i128_to_double(const int64_t* hi, const uint64_t* lo, double* out, int64_t count, void* stream) {
  BF_API_BEGIN
  cudaStream_t s = (cudaStream_t)stream;
  InStage hs(hi, 8 * count, s), ls(lo, 8 * count, s);
  OutStage os(out, 8 * count, s);
  i128_impl((const int64_t*)hs.dptr, (const uint64_t*)ls.dptr, (double*)os.dptr, count, s);
  os.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_API_END
}

int bf_fixed_point(const double* y, int64_t n, int64_t sampsize, int64_t* yq, int32_t* q, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(y && yq && q && n >= 1, BF_EINVAL, "bf_fixed_point: bad args");
  cudaStream_t s = (cudaStream_t)stream;
  InStage ys(y, 8 * n, s);
  OutStage os(yq, 8 * n, s);
  fixed_point_impl((const double*)ys.dptr, n, sampsize ? sampsize : n, (int64_t*)os.dptr, q, s);
  os.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_API_END
}

int bf_bootstrap(uint64_t seed, int32_t t0, int32_t ntrees, int64_t n, int64_t sampsize, int32_t replace,
                 int32_t* w, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(w && n >= 1 && ntrees >= 0 && t0 >= 0, BF_EINVAL, "bf_bootstrap: bad args");
  cudaStream_t s = (cudaStream_t)stream;
  int64_t ss = sampsize ? sampsize : n;
  BF_REQUIRE(replace || ss == n, BF_ENOTIMPL, "bf_bootstrap: replace=0 needs sampsize == n");
  OutStage ws(w, sizeof(int32_t) * n * ntrees, s);
  bootstrap_impl(seed, t0, ntrees, n, ss, replace, (int32_t*)ws.dptr, s);
  ws.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_API_END
}

int bf_perm(uint64_t seed, int32_t t, int32_t m, int64_t n_o, int64_t* out, void* stream) {
  BF_API_BEGIN
  BF_REQUIRE(out && n_o >= 1, BF_EINVAL, "bf_perm: bad args");
  cudaStream_t s = (cudaStream_t)stream;
  OutStage os(out, 8 * n_o, s);
  perm_impl(seed, t, m, n_o, (int64_t*)os.dptr, s);
  os.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_API_END
}

}  // extern "C"

// ------------------------------------------------------------------ measurement hooks
#include <atomic>
#include <map>

namespace bf {
namespace {
struct PendingEv {
  const char* name;
  cudaEvent_t a, b;
  double bytes;
  int launches;
};
std::mutex g_prof_mu;
bool g_prof_on = false;
std::atomic<int64_t> g_launches{0};
std::vector<PendingEv> g_pending;
std::vector<cudaEvent_t> g_ev_pool;
struct Tot {
  double ms = 0, bytes = 0;
  int64_t launches = 0;
};
std::map<std::string, Tot> g_tot;

cudaEvent_t ev_get() {
  if (!g_ev_pool.empty()) {
    cudaEvent_t e = g_ev_pool.back();
    g_ev_pool.pop_back();
    return e;
  }
  cudaEvent_t e;
  cudaEventCreate(&e);
  return e;
}

void drain_locked() {
  for (auto& p : g_pending) {
    cudaEventSynchronize(p.b);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, p.a, p.b);
    Tot& t = g_tot[p.name];
    t.ms += ms;
    t.bytes += p.bytes;
    t.launches += p.launches;
    g_ev_pool.push_back(p.a);
    g_ev_pool.push_back(p.b);
  }
  g_pending.clear();
}
}  // namespace

KScope::KScope(const char* nm, cudaStream_t st, double by, int nl) : s(st) {
  g_launches += nl;
  if (!g_prof_on) return;
  std::lock_guard<std::mutex> lk(g_prof_mu);
  name = nm;
  bytes = by;
  launches = nl;
  a = ev_get();
  b = ev_get();
  cudaEventRecord(a, st);
  active = true;
}

KScope::~KScope() {
  if (!active) return;
  std::lock_guard<std::mutex> lk(g_prof_mu);
  cudaEventRecord(b, s);
  g_pending.push_back(PendingEv{name, a, b, bytes, launches});
  if (g_pending.size() > 8192) drain_locked();  // bounded: waits for recorded pairs
}
bool prof_enabled() { return g_prof_on; }

void prof_add_bytes(const char* name, double bytes) {
  if (!g_prof_on) return;
  std::lock_guard<std::mutex> lk(g_prof_mu);
  g_tot[name].bytes += bytes;
}
}  // namespace bf

extern "C" {
int bf_profile_enable(int on) {
  std::lock_guard<std::mutex> lk(bf::g_prof_mu);
  bf::g_prof_on = on != 0;
  return BF_OK;
}

int bf_profile_read(bf_kernel_stat* stats, int cap, int* count) {
  std::lock_guard<std::mutex> lk(bf::g_prof_mu);
  bf::drain_locked();
  int k = 0;
  for (auto& kv : bf::g_tot) {
    if (stats && k < cap) {
      memset(stats[k].name, 0, sizeof(stats[k].name));
      strncpy(stats[k].name, kv.first.c_str(), sizeof(stats[k].name) - 1);
      stats[k].ms = kv.second.ms;
      stats[k].launches = kv.second.launches;
      stats[k].bytes = kv.second.bytes;
    }
    ++k;
  }
  if (count) *count = k;
  if (stats) bf::g_tot.clear();
  return BF_OK;
}

int64_t bf_launch_count(void) { return bf::g_launches.load(); }
}
