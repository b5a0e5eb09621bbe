// bf_internal.cuh -- internal declarations of the B200 BlackForest library.
//
// Device primitives (Philox4x32-10, 64-bit mulhi, correctly rounded int128 ->
// double, the exact split key) are written here from DESIGN.md S1-S4; nothing
// is shared with oracle/ (the CPU oracle is independent test infrastructure).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/bf.h"

namespace bf {

// ------------------------------------------------------------------ errors
struct Error {
  int code;
  std::string msg;
};
void set_error(const std::string& m);
#define BF_CUDA_CHECK(expr)                                                                   \
  do {                                                                                        \
    cudaError_t e_ = (expr);                                                                  \
    if (e_ != cudaSuccess)                                                                    \
      throw ::bf::Error{BF_ECUDA, std::string(#expr " -> ") + cudaGetErrorString(e_) + " @" + \
                                      __FILE__ + ":" + std::to_string(__LINE__)};             \
  } while (0)
#define BF_REQUIRE(cond, code, m) \
  do {                            \
    if (!(cond)) throw ::bf::Error{(code), (m)}; \
  } while (0)

// ------------------------------------------------------------------ memory
void* dev_alloc(size_t bytes, cudaStream_t s);
int64_t memory_budget();  // bf_set_memory_budget (0: ask the driver)
void dev_free(void* p, cudaStream_t s);

template <class T>
struct DBuf {  // stream-ordered device buffer (RAII)
  T* p = nullptr;
  size_t n = 0;
  cudaStream_t s = nullptr;
  DBuf() = default;
  DBuf(size_t count, cudaStream_t st) { alloc(count, st); }
  void alloc(size_t count, cudaStream_t st) {
    release();
    s = st;
    n = count;
    if (count) p = static_cast<T*>(dev_alloc(count * sizeof(T), st));
  }
  void release() {
    if (p) dev_free(p, s);
    p = nullptr;
    n = 0;
  }
  ~DBuf() { release(); }
  DBuf(const DBuf&) = delete;
  DBuf& operator=(const DBuf&) = delete;
  DBuf(DBuf&& o) noexcept : p(o.p), n(o.n), s(o.s) { o.p = nullptr; o.n = 0; }
  DBuf& operator=(DBuf&& o) noexcept {
    if (this != &o) { release(); p = o.p; n = o.n; s = o.s; o.p = nullptr; o.n = 0; }
    return *this;
  }
  size_t bytes() const { return n * sizeof(T); }
};

// Host/device pointer staging: a host input is copied to a temporary device
// buffer on the stream; a host output is copied back at finish().
bool is_device_ptr(const void* p);

struct InStage {
  const void* dptr = nullptr;
  DBuf<char> tmp;
  InStage(const void* ptr, size_t bytes, cudaStream_t s);
};
struct OutStage {
  void* dptr = nullptr;
  void* host = nullptr;
  size_t bytes = 0;
  DBuf<char> tmp;
  OutStage(void* ptr, size_t bytes, cudaStream_t s);
  void finish(cudaStream_t s);  // D2H if host (caller synchronises)
};

// ------------------------------------------------------------------ measurement
// Scope around ONE logical launch (a kernel, or a CUB call): counts it and,
// when profiling is enabled, brackets it with a CUDA event pair.
struct KScope {
  KScope(const char* name, cudaStream_t s, double bytes, int launches = 1);
  ~KScope();
  KScope(const KScope&) = delete;
  KScope& operator=(const KScope&) = delete;
  cudaStream_t s;
  bool active = false;
  const char* name = nullptr;
  double bytes = 0;
  int launches = 0;
  cudaEvent_t a = nullptr, b = nullptr;
};

// Adds algorithmic bytes to a kernel class after the fact (sizes known only
// after a device->host summary read).
void prof_add_bytes(const char* name, double bytes);
bool prof_enabled();

// ------------------------------------------------------------------ device primitives
// S1: Philox4x32-10.
__host__ __device__ __forceinline__ void philox4x32_10(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                                                       uint32_t k0, uint32_t k1, uint32_t out[4]) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
#ifdef __CUDA_ARCH__
    const uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
#else
    const uint64_t p0 = (uint64_t)0xD2511F53u * c0, p1 = (uint64_t)0xCD9E8D57u * c2;
    const uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    const uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
#endif
    const uint32_t n0 = hi1 ^ c1 ^ k0, n2 = hi0 ^ c3 ^ k1;
    c0 = n0;
    c1 = lo1;
    c2 = n2;
    c3 = lo0;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  out[0] = c0;
  out[1] = c1;
  out[2] = c2;
  out[3] = c3;
}

__device__ __forceinline__ void philox_u64x2(uint64_t seed, uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                                             uint64_t& u0, uint64_t& u1) {
  uint32_t x[4];
  philox4x32_10(c0, c1, c2, c3, (uint32_t)seed, (uint32_t)(seed >> 32), x);
  u0 = (uint64_t)x[0] | ((uint64_t)x[1] << 32);
  u1 = (uint64_t)x[2] | ((uint64_t)x[3] << 32);
}

__device__ __forceinline__ uint64_t mulhi64(uint64_t u, uint64_t r) { return __umul64hi(u, r); }

// S3 KEY stream: child key of node key K.
__device__ __forceinline__ uint64_t child_key(uint64_t seed, uint32_t t, uint64_t K, uint32_t side) {
  uint64_t u0, u1;
  philox_u64x2(seed, (uint32_t)K, (uint32_t)(K >> 32), t, 0x40000000u | side, u0, u1);
  return u0;
}

// Correctly rounded (nearest-even) conversion of a signed 128-bit integer.
// The top 64 significant bits are converted by __ull2double_rn with the
// remaining bits folded into the LSB as a sticky bit (the LSB lies below the
// rounding position because the top word has its MSB set), then scaled by an
// exact power of two.
__device__ __forceinline__ double i128_to_double(__int128 v) {
  const bool neg = v < 0;
  unsigned __int128 u = neg ? (unsigned __int128)(-(v + 1)) + 1u : (unsigned __int128)v;
  const uint64_t hi = (uint64_t)(u >> 64), lo = (uint64_t)u;
  double d;
  if (hi == 0) {
    d = __ull2double_rn(lo);
  } else {
    const int lz = __clzll(hi);
    const uint64_t m = lz ? ((hi << lz) | (lo >> (64 - lz))) : hi;
    const uint64_t rest = lo << lz;  // lz < 64
    d = __ull2double_rn(m | (rest != 0 ? 1ull : 0ull));
    const double scale = __longlong_as_double((long long)(1023 + 64 - lz) << 52);  // 2^(64-lz)
    d = __dmul_rn(d, scale);
  }
  return neg ? -d : d;
}

// S4.3 exact split key: g = RN(RN(RN(D)^2) / RN(n_l*n_r)), D = n_k*S_l - n_l*S_k.
__device__ __forceinline__ double split_key(int64_t nk, int64_t Sk, int64_t nl, int64_t Sl) {
  const __int128 D = (__int128)nk * (__int128)Sl - (__int128)nl * (__int128)Sk;
  const double d = i128_to_double(D);
  const double nn = __ll2double_rn(nl * (nk - nl));
  return __ddiv_rn(__dmul_rn(d, d), nn);
}

__device__ __forceinline__ double canon(double x) { return __dadd_rn(x, 0.0); }  // -0 -> +0 (R18)

// S4.6 threshold inside the gap [a, b).
__device__ __forceinline__ double split_threshold(double a, double b) {
  double t = __dadd_rn(__dmul_rn(0.5, a), __dmul_rn(0.5, b));
  if (!(t < b)) t = a;
  if (t < a) t = a;
  return t;
}

// ------------------------------------------------------------------ forest
struct Node16 {  // packed node for traversal: 16 B, one sector-aligned load
  double v;       // threshold (internal) or leaf value
  int32_t feature;  // -1 leaf
  int32_t left;     // local id of the left child; right = left + 1
};
static_assert(sizeof(Node16) == 16, "Node16 must be 16 bytes");

// Compact traversal node (predict.cu k_pack8; layout documented there): internal = {float thr, LL<<31 |
// RL<<30 | feature<<22 | rel}, leaf = the fp64 value; roots8[t] = root id | ROOT_LEAF for one-node trees.
constexpr int N8_FEAT_BITS = 8, N8_REL_BITS = 22;
constexpr uint32_t ROOT_LEAF = 0x80000000u;
__device__ __forceinline__ double leaf8(uint2 v) { return __hiloint2double((int)v.y, (int)v.x); }
__device__ __forceinline__ uint32_t n8_feature(uint2 w) { return (w.y >> N8_REL_BITS) & ((1u << N8_FEAT_BITS) - 1u); }
__device__ __forceinline__ uint32_t n8_rel(uint2 w) { return w.y & ((1u << N8_REL_BITS) - 1u); }
// Two-level 32-byte groups (predict.cu g32_get; layout documented there): one 256-bit read-only load per group.
constexpr uint32_t G32_LEAF = 0x80000000u;  // walk state: the slot being loaded is a leaf
__device__ __forceinline__ ulonglong4 ldg256(const ulonglong4* p) {
  ulonglong4 v;
  asm volatile("ld.global.nc.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(v.x), "=l"(v.y), "=l"(v.z), "=l"(v.w) : "l"(p));
  return v;
}

}  // namespace bf

struct bf_forest {
  bf_forest_info info;
  std::vector<int64_t> tree_off;  // host copy, ntrees + 1
  int64_t* d_tree_off = nullptr;
  bf::Node16* d_nodes = nullptr;
  int32_t* d_count = nullptr;
  double* d_value = nullptr;
  double* d_drss = nullptr;
  // Compact 8-byte traversal copy of d_nodes (predict.cu, built on first use):
  // 0 not built, 1 built, -1 not representable (p > 256, >= 2^31 nodes, or a child stored before its parent).
  uint2* d_nodes8 = nullptr;
  uint32_t* d_roots8 = nullptr;  // per tree: global root id | 1<<31 if the tree is a single leaf
  int nodes8_state = 0;
  // Two-level 32-byte groups (predict.cu g32_get, built on first use; same states as nodes8_state): a group holds
  // an internal node at even depth and its two children, so one 256-bit load decides two levels of a walk.
  ulonglong4* d_g32 = nullptr;
  uint32_t* d_g32_root = nullptr;  // per tree: global slot of the root | ROOT_LEAF if the tree is a single leaf
  std::vector<int64_t> g32_off;    // host: first slot of each tree, ntrees + 1
  int g32_state = 0;
  int device = 0;
  cudaStream_t stream = nullptr;       // stream the forest's memory was allocated on (freed stream-ordered on it)
  mutable bool foreign_stream = false;  // some call used the forest on another stream (free waits for the device)
  void touch(cudaStream_t s) const {
    if (s != stream) foreign_stream = true;
  }
};

namespace bf {
void forest_alloc(bf_forest* f, int64_t total_nodes, int32_t ntrees, cudaStream_t s);
void forest_release(bf_forest* f);

// prims.cu: hand-written scans, LSD radix sort, unique (no library kernels on the path)
void scan_exclusive(const uint64_t* in, uint64_t* out, int64_t n, cudaStream_t s);
void scan_exclusive(const int32_t* in, int32_t* out, int64_t n, cudaStream_t s);
void scan_exclusive(const uint32_t* in, uint32_t* out, int64_t n, cudaStream_t s);
void scan_inclusive(const uint32_t* in, uint32_t* out, int64_t n, cudaStream_t s);
// Sorts nseg equal-length segments of n keys (k0[seg * n + i]) independently, ascending and stable, with
// optional 32-bit values (v0/v1 NULL: keys only); k1 / v1 are scratch of the same size.  Returns the buffer
// that holds the sorted keys (k0 or k1); *vals_out the one with the values.
const uint64_t* radix_sort_u64(uint64_t* k0, uint64_t* k1, uint32_t* v0, uint32_t* v1, int64_t n, int nseg,
                               cudaStream_t s, uint32_t** vals_out);
// Distinct values of sorted keys, in order; *count_dev (device int32) = how many.
void unique_u64(const uint64_t* sorted, int64_t n, uint64_t* out, int32_t* count_dev, cudaStream_t s);

// fit.cu
bool release_list_workspace();  // false while a fit holds it
void fit_impl(const double* X, int64_t ldx, const double* y, int64_t n, int32_t p, const bf_params& prm,
              cudaStream_t s, bf_forest** out);
void fixed_point_impl(const double* y, int64_t n, int64_t sampsize, int64_t* yq, int32_t* q, cudaStream_t s);
void bootstrap_impl(uint64_t seed, int32_t t0, int32_t ntrees, int64_t n, int64_t sampsize, int32_t replace,
                    int32_t* w, cudaStream_t s);
// predict.cu
const uint2* nodes8_get(bf_forest* f, cudaStream_t s);  // NULL if not representable
const ulonglong4* g32_get(bf_forest* f, cudaStream_t s);  // NULL if not representable
void predict_impl(const bf_forest* f, const double* Xq, int64_t ldq, int64_t m, double* yhat_sum, double* yhat,
                  int32_t ntree_total, cudaStream_t s);
void pd_grid_impl(const double* x, int64_t n, int32_t n_pt, double* grid, int32_t* G_host, cudaStream_t s);
void partial_dependence_impl(const bf_forest* f, const double* X, int64_t ldx, int64_t n, int32_t m,
                             const double* grid, int32_t G, double* pd_sum, double* pd, int32_t ntree_total,
                             cudaStream_t s);
// importance.cu
// row-major RN_f32 copy of a column-major fp64 matrix (stride xfs floats, a multiple of 4, zero padded)
void xf_rows_impl(const double* X, int64_t ldx, int64_t n, int p, float* Xf, int xfs, cudaStream_t s);
void oob_importance_impl(const bf_forest* f, const double* X, int64_t ldx, const double* y, int64_t n, int32_t p,
                         const bf_oob_accum& acc, cudaStream_t s);
void importance_finalize_impl(const double* d_slots, const double* npur_slots, const double* oob_sum,
                              const int32_t* oob_cnt, const double* y, int64_t n, int32_t p, int32_t ntree,
                              double* out_p4 /* 4*p: inc, raw, sd, npur */, double* out_s2, cudaStream_t s);
void perm_impl(uint64_t seed, int32_t t, int32_t m, int64_t n_o, int64_t* out, cudaStream_t s);
// pca.cu
void pca_retained_impl(const double* sdev, int32_t p, double frac, int32_t cap, int32_t* k_host, cudaStream_t s);
void pca_impl(const double* X, int64_t ldx, int64_t n, int32_t p, int32_t scale, int32_t k, double* sdev,
              double* rotation, double* center, double* scores, cudaStream_t s);
void varimax_impl(const double* L, int64_t ldl, int32_t p, int32_t k, int32_t normalize, double eps, double* loadings,
                  double* rotmat, int32_t* iters_host, cudaStream_t s);
// models.cu
void glm_gaussian_impl(const double* Z, int64_t ldz, int64_t n, int32_t k, const double* Y, int64_t ldy, int32_t r,
                       double* coef, double* deviance, double* null_deviance, cudaStream_t s);
void glm_predict_impl(const double* Z, int64_t ldz, int64_t n, int32_t k, const double* coef, int32_t r, double* out,
                      int64_t ldo, cudaStream_t s);
void mars_fit_impl(const double* X, int64_t ldx, int64_t n, int32_t d, const double* y, int32_t nk, double thresh,
                   double penalty, int32_t* nterms, int32_t* tvar, double* tknot, int32_t* tdir, double* coef,
                   double* stats, cudaStream_t s);
void mars_predict_impl(const double* X, int64_t ldx, int64_t m, int32_t d, int32_t nt, const int32_t* tvar,
                       const double* tknot, const int32_t* tdir, const double* coef, double* out, cudaStream_t s);
void rank_similarity_impl(const double* a, const double* b, int32_t p, double* out, cudaStream_t s);
void log_size_design_impl(const double* size, int64_t n, double* Z, int64_t ldz, cudaStream_t s);
void prediction_error_impl(const double* yhat, const double* y, int64_t m, double* out_host, cudaStream_t s);
// misc kernels (capi.cu)
void philox_impl(const uint32_t* ctr, uint32_t k0, uint32_t k1, uint32_t* out, int64_t count, cudaStream_t s);
void i128_impl(const int64_t* hi, const uint64_t* lo, double* out, int64_t count, cudaStream_t s);

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Largest dynamic shared memory a launch of `func` may request (opt-in limit
// minus the kernel's static shared memory); sets the attribute accordingly.
template <class F>
int dyn_smem_limit(F func) {
  int dev = 0, optin = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, (const void*)func);
  const int lim = optin - (int)fa.sharedSizeBytes;
  cudaFuncSetAttribute((const void*)func, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
  return lim;
}
}  // namespace bf
