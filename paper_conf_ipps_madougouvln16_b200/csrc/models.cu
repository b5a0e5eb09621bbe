// models.cu -- counter models and the platform-similarity statistic
// (readings R26, R27).
//
// bf_glm_gaussian ("(generalized) linear models are sufficient",
// P:173, "generalized linear models ... low residual deviance"): R glm
// with the default gaussian family = least squares of every response column
// on one shared design Z (n x k).  Solved by column-scaled CholeskyQR2, never
// forming Q: with D = diag(1/||Z_j||), R1 = chol(D Z^T Z D), W1 = D R1^-1,
// R2 = chol((Z W1)^T (Z W1)), W = W1 R2^-1, the columns of Q = Z W are
// orthonormal to working precision and coef = W (Q^T Y).  The residual and
// null deviances are then summed directly over the rows.  All cross products
// are per-CTA partial sums over row blocks, reduced in a fixed order
// (deterministic); the k x k factorisations run in one CTA in fp64.
//
// bf_rank_similarity ("the same variable importance ranking"):
// Spearman's rho on mid-ranks and Kendall's tau-b, O(p^2) pair counts in
// exact integers in one CTA.
#include <algorithm>
#include <cmath>

#include "bf_internal.cuh"

namespace bf {
namespace {

constexpr int GT = 256;       // threads of the cross-product CTAs
constexpr int GROWS = 32;     // rows staged per iteration
constexpr int GMAXK = 32;     // design columns
constexpr int GMAXR = 64;     // responses per call
constexpr int GACC = (GMAXK * (GMAXK + GMAXR) + GT - 1) / GT;  // accumulators per thread

// partial[blk][a][c] = sum over the CTA's rows of q_a * b_c, q = z W (W = NULL: q = z),
// b = [q | y] (c < k: q_c, else y_{c-k}); kb = k + r columns on the right.
__global__ void __launch_bounds__(GT) k_glm_cross(const double* __restrict__ Z, int64_t ldz, int64_t n, int k,
                                                  const double* __restrict__ W, const double* __restrict__ Y,
                                                  int64_t ldy, int r, double* __restrict__ partial) {
  __shared__ double sq[GROWS][GMAXK + 1];
  __shared__ double sy[GROWS][GMAXR + 1];
  __shared__ double sw[GMAXK * GMAXK];
  const int tid = threadIdx.x;
  const int kb = k + r;
  if (W)
    for (int i = tid; i < k * k; i += GT) sw[i] = W[i];
  double acc[GACC];
#pragma unroll
  for (int u = 0; u < GACC; ++u) acc[u] = 0.0;
  __syncthreads();
  for (int64_t r0 = (int64_t)blockIdx.x * GROWS; r0 < n; r0 += (int64_t)gridDim.x * GROWS) {
    const int rows = (int)(n - r0 < GROWS ? n - r0 : GROWS);
    // stage z (then q = z W in place, row by row) and y
    for (int i = tid; i < GROWS * k; i += GT) {
      const int rr = i % GROWS, c = i / GROWS;
      sq[rr][c] = rr < rows ? Z[(int64_t)c * ldz + r0 + rr] : 0.0;
    }
    for (int i = tid; i < GROWS * r; i += GT) {
      const int rr = i % GROWS, c = i / GROWS;
      sy[rr][c] = rr < rows ? Y[(int64_t)c * ldy + r0 + rr] : 0.0;
    }
    __syncthreads();
    if (W) {
      double qv[GMAXK];
      const int rr = tid % GROWS, part = tid / GROWS;  // GT / GROWS threads per row: columns part, part + 8, ...
      for (int c = part; c < k; c += GT / GROWS) {
        double s = 0.0;
        for (int a = 0; a <= c; ++a) s += sq[rr][a] * sw[c * k + a];  // W upper triangular (column-major)
        qv[c / (GT / GROWS)] = s;
      }
      __syncthreads();
      for (int c = part; c < k; c += GT / GROWS) sq[rr][c] = qv[c / (GT / GROWS)];
      __syncthreads();
    }
#pragma unroll
    for (int u = 0; u < GACC; ++u) {
      const int e = tid + u * GT;
      if (e < k * kb) {
        const int a = e % k, c = e / k;
        double s = 0.0;
        if (c < k)
          for (int rr = 0; rr < rows; ++rr) s += sq[rr][a] * sq[rr][c];
        else
          for (int rr = 0; rr < rows; ++rr) s += sq[rr][a] * sy[rr][c - k];
        acc[u] += s;
      }
    }
    __syncthreads();
  }
#pragma unroll
  for (int u = 0; u < GACC; ++u) {
    const int e = tid + u * GT;
    if (e < k * kb) partial[(int64_t)blockIdx.x * k * kb + e] = acc[u];
  }
}

// out[e] = sum over blocks (fixed order) of partial[blk][e]
__global__ void k_reduce_partials(const double* __restrict__ partial, int nblk, int ne, double* __restrict__ out) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= ne) return;
  double s = 0.0;
  for (int b = 0; b < nblk; ++b) s += partial[(int64_t)b * ne + e];
  out[e] = s;
}

// One CTA: from C = cross[k x (k + r)] (column-major, ld k) of q = z W_in:
//   first pass (W_in == NULL): D = diag(1/sqrt(C_jj)), G = D C D, W_base = D;
//   later passes: G = C, W_base = W_in.
// R = chol(G) (upper), W_out = W_base R^-1.  status = 1 if G is not positive definite
// to working precision (rank-deficient design).
__global__ void k_glm_chol(const double* __restrict__ C, int k, const double* __restrict__ W_in,
                           double* __restrict__ W_out, int* status) {
  __shared__ double G[GMAXK * GMAXK], R[GMAXK * GMAXK], Ri[GMAXK * GMAXK], Wb[GMAXK * GMAXK], d[GMAXK];
  const int tid = threadIdx.x;
  for (int i = tid; i < k; i += blockDim.x) d[i] = W_in ? 1.0 : (C[i * k + i] > 0.0 ? 1.0 / sqrt(C[i * k + i]) : 0.0);
  __syncthreads();
  for (int e = tid; e < k * k; e += blockDim.x) {
    const int i = e % k, j = e / k;
    G[e] = C[e] * d[i] * d[j];
    Wb[e] = W_in ? W_in[e] : (i == j ? d[i] : 0.0);
    R[e] = 0.0;
    Ri[e] = 0.0;
  }
  __syncthreads();
  if (tid == 0) {
    bool ok = true;
    for (int j = 0; j < k && ok; ++j) {  // R^T R = G, column by column
      for (int i = 0; i < j; ++i) {
        double s = G[j * k + i];
        for (int l = 0; l < i; ++l) s -= R[i * k + l] * R[j * k + l];
        R[j * k + i] = s / R[i * k + i];
      }
      double s = G[j * k + j];
      for (int l = 0; l < j; ++l) s -= R[j * k + l] * R[j * k + l];
      if (!(s > 1e-13 * G[j * k + j]) || d[j] == 0.0) ok = false;  // scaled design: G_jj ~ 1
      R[j * k + j] = ok ? sqrt(s) : 1.0;
    }
    if (!ok) *status = 1;
    for (int j = 0; j < k; ++j) {  // Ri = R^-1 (upper), column j by back substitution
      Ri[j * k + j] = 1.0 / R[j * k + j];
      for (int i = j - 1; i >= 0; --i) {
        double s = 0.0;
        for (int l = i + 1; l <= j; ++l) s += R[l * k + i] * Ri[j * k + l];
        Ri[j * k + i] = -s / R[i * k + i];
      }
    }
  }
  __syncthreads();
  for (int e = tid; e < k * k; e += blockDim.x) {  // W_out = Wb Ri (both upper triangular)
    const int i = e % k, j = e / k;
    double s = 0.0;
    for (int l = i; l <= j; ++l) s += Wb[l * k + i] * Ri[j * k + l];
    W_out[e] = i <= j ? s : 0.0;
  }
}

// coef (k x r, ld k) = W d, d = (Q^T Y) = columns k.. of the cross product of q = z W.
__global__ void k_glm_coef(const double* __restrict__ C, const double* __restrict__ W, int k, int r,
                           double* __restrict__ coef) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= k * r) return;
  const int i = e % k, j = e / k;
  double s = 0.0;
  for (int l = i; l < k; ++l) s += W[l * k + i] * C[(int64_t)(k + j) * k + l];
  coef[e] = s;
}

// per CTA partials of sum y (pass 0) or of [sum (y - mean)^2, sum (y - z c)^2] (pass 1), per response.
__global__ void __launch_bounds__(GT) k_glm_dev(const double* __restrict__ Z, int64_t ldz, int64_t n, int k,
                                                const double* __restrict__ Y, int64_t ldy, int r,
                                                const double* __restrict__ coef, const double* __restrict__ mean,
                                                int pass, double* __restrict__ partial) {
  __shared__ double sc[GMAXK * GMAXR];
  __shared__ double red[GT / 32][2];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  if (pass == 1)
    for (int i = tid; i < k * r; i += GT) sc[i] = coef[i];
  __syncthreads();
  for (int j = 0; j < r; ++j) {
    double s0 = 0.0, s1 = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * GT + tid; i < n; i += (int64_t)gridDim.x * GT) {
      const double yv = Y[(int64_t)j * ldy + i];
      if (pass == 0) {
        s0 += yv;
      } else {
        const double dm = yv - mean[j];
        s0 += dm * dm;
        double f = 0.0;
        for (int a = 0; a < k; ++a) f += Z[(int64_t)a * ldz + i] * sc[j * k + a];
        const double e = yv - f;
        s1 += e * e;
      }
    }
    for (int o = 16; o > 0; o >>= 1) {
      s0 += __shfl_down_sync(0xffffffffu, s0, o);
      s1 += __shfl_down_sync(0xffffffffu, s1, o);
    }
    if (lane == 0) {
      red[wid][0] = s0;
      red[wid][1] = s1;
    }
    __syncthreads();
    if (tid == 0) {
      double t0 = 0.0, t1 = 0.0;
      for (int w = 0; w < GT / 32; ++w) {
        t0 += red[w][0];
        t1 += red[w][1];
      }
      partial[((int64_t)blockIdx.x * r + j) * 2] = t0;
      partial[((int64_t)blockIdx.x * r + j) * 2 + 1] = t1;
    }
    __syncthreads();
  }
}

__global__ void k_glm_dev_final(const double* __restrict__ partial, int nblk, int r, int64_t n, int pass,
                                double* __restrict__ mean, double* __restrict__ dev, double* __restrict__ null_dev) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= r) return;
  double t0 = 0.0, t1 = 0.0;
  for (int b = 0; b < nblk; ++b) {
    t0 += partial[((int64_t)b * r + j) * 2];
    t1 += partial[((int64_t)b * r + j) * 2 + 1];
  }
  if (pass == 0) {
    mean[j] = t0 / (double)n;
  } else {
    null_dev[j] = t0;
    dev[j] = t1;
  }
}

// ------------------------------------------------------------------ rank similarity (R27)
constexpr int RT = 256;
__global__ void __launch_bounds__(RT) k_rank_similarity(const double* __restrict__ a, const double* __restrict__ b,
                                                        int p, double* __restrict__ out) {
  extern __shared__ double rsm[];  // ra[p], rb[p]
  double* ra = rsm;
  double* rb = rsm + p;
  __shared__ unsigned long long cnt[RT / 32][4];
  __shared__ double red[RT / 32][3];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  unsigned long long C = 0, D = 0, Ta = 0, Tb = 0;
  for (int i = tid; i < p; i += RT) {
    const double ai = a[i], bi = b[i];
    long long la = 0, ea = 0, lb = 0, eb = 0;
    for (int j = 0; j < p; ++j) {
      const double aj = a[j], bj = b[j];
      la += aj < ai;
      ea += aj == ai;
      lb += bj < bi;
      eb += bj == bi;
      if (j > i) {
        const bool za = aj == ai, zb = bj == bi;
        if (za && zb) continue;
        if (za)
          ++Ta;
        else if (zb)
          ++Tb;
        else if ((ai > aj) == (bi > bj))
          ++C;
        else
          ++D;
      }
    }
    ra[i] = (double)la + (double)(ea + 1) * 0.5;  // mid-ranks (exact: halves of integers)
    rb[i] = (double)lb + (double)(eb + 1) * 0.5;
  }
  for (int o = 16; o > 0; o >>= 1) {
    C += __shfl_down_sync(0xffffffffu, C, o);
    D += __shfl_down_sync(0xffffffffu, D, o);
    Ta += __shfl_down_sync(0xffffffffu, Ta, o);
    Tb += __shfl_down_sync(0xffffffffu, Tb, o);
  }
  if (lane == 0) {
    cnt[wid][0] = C;
    cnt[wid][1] = D;
    cnt[wid][2] = Ta;
    cnt[wid][3] = Tb;
  }
  __syncthreads();
  // Pearson of the mid-ranks: the mean of 1..p mid-ranks is exactly (p + 1) / 2
  const double mr = 0.5 * (double)(p + 1);
  double sab = 0.0, saa = 0.0, sbb = 0.0;
  for (int i = tid; i < p; i += RT) {
    const double da = ra[i] - mr, db = rb[i] - mr;
    sab += da * db;
    saa += da * da;
    sbb += db * db;
  }
  for (int o = 16; o > 0; o >>= 1) {
    sab += __shfl_down_sync(0xffffffffu, sab, o);
    saa += __shfl_down_sync(0xffffffffu, saa, o);
    sbb += __shfl_down_sync(0xffffffffu, sbb, o);
  }
  if (lane == 0) {
    red[wid][0] = sab;
    red[wid][1] = saa;
    red[wid][2] = sbb;
  }
  __syncthreads();
  if (tid == 0) {
    unsigned long long c = 0, d = 0, ta = 0, tb = 0;
    double s0 = 0.0, s1 = 0.0, s2 = 0.0;
    for (int w = 0; w < RT / 32; ++w) {
      c += cnt[w][0];
      d += cnt[w][1];
      ta += cnt[w][2];
      tb += cnt[w][3];
      s0 += red[w][0];
      s1 += red[w][1];
      s2 += red[w][2];
    }
    const double den_s = sqrt(s1 * s2);
    out[0] = den_s > 0.0 ? s0 / den_s : nan("");
    const double den_k = sqrt((double)(c + d + ta) * (double)(c + d + tb));
    out[1] = den_k > 0.0 ? ((double)c - (double)d) / den_k : nan("");
  }
}

// out[j * ldo + i] = sum_a Z[a * ldz + i] * coef[j * k + a]: the counter models evaluated on new rows.
__global__ void k_glm_predict(const double* __restrict__ Z, int64_t ldz, int64_t n, int k,
                              const double* __restrict__ coef, int r, double* __restrict__ out, int64_t ldo) {
  __shared__ double sc[GMAXK * GMAXR];
  for (int i = threadIdx.x; i < k * r; i += blockDim.x) sc[i] = coef[i];
  __syncthreads();
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  double z[GMAXK];
#pragma unroll 8
  for (int a = 0; a < k; ++a) z[a] = Z[(int64_t)a * ldz + i];
  for (int j = 0; j < r; ++j) {
    double f = 0.0;
    for (int a = 0; a < k; ++a) f += z[a] * sc[j * k + a];
    out[(int64_t)j * ldo + i] = f;
  }
}

}  // namespace

void glm_predict_impl(const double* Z_in, int64_t ldz, int64_t n, int32_t k, const double* coef_in, int32_t r,
                      double* out_in, int64_t ldo, cudaStream_t s) {
  BF_REQUIRE(k >= 1 && k <= GMAXK && r >= 1 && r <= GMAXR && n >= 0, BF_EINVAL,
             "bf_glm_predict: need 1 <= k <= 32, 1 <= r <= 64, n >= 0");
  if (n == 0) return;
  InStage Zs(Z_in, sizeof(double) * (size_t)(ldz * (k - 1) + n), s), cs(coef_in, sizeof(double) * (size_t)k * r, s);
  OutStage os(out_in, sizeof(double) * (size_t)(ldo * (r - 1) + n), s);
  {
    KScope ks_("k_glm_predict", s, 8.0 * (double)n * (k + r));
    k_glm_predict<<<(unsigned)ceil_div(n, 128), 128, 0, s>>>((const double*)Zs.dptr, ldz, n, k,
                                                            (const double*)cs.dptr, r, (double*)os.dptr, ldo);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  os.finish(s);
  if (os.host || Zs.tmp.p || cs.tmp.p) BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

void glm_gaussian_impl(const double* Z_in, int64_t ldz, int64_t n, int32_t k, const double* Y_in, int64_t ldy,
                       int32_t r, double* coef_in, double* dev_in, double* null_in, cudaStream_t s) {
  BF_REQUIRE(k >= 1 && k <= GMAXK && r >= 1 && r <= GMAXR && n >= k, BF_EINVAL,
             "bf_glm_gaussian: need 1 <= k <= 32, 1 <= r <= 64, n >= k");
  InStage Zs(Z_in, sizeof(double) * (size_t)(ldz * (k - 1) + n), s);
  InStage Ys(Y_in, sizeof(double) * (size_t)(ldy * (r - 1) + n), s);
  OutStage cs(coef_in, sizeof(double) * (size_t)k * r, s), ds(dev_in, dev_in ? sizeof(double) * r : 0, s),
      ns(null_in, null_in ? sizeof(double) * r : 0, s);
  const double* Z = (const double*)Zs.dptr;
  const double* Y = (const double*)Ys.dptr;
  int dev_id = 0, nsm = 148;
  cudaGetDevice(&dev_id);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev_id);
  const int nblk = (int)std::max<int64_t>(1, std::min<int64_t>(2 * nsm, ceil_div(n, GROWS)));
  const int kb = k + r;
  DBuf<double> part((size_t)nblk * k * kb, s), cross((size_t)k * kb, s), W1((size_t)k * k, s), W((size_t)k * k, s),
      dpart((size_t)nblk * r * 2, s), mean(r, s), tdev, tnull;
  DBuf<int> status(1, s);
  BF_CUDA_CHECK(cudaMemsetAsync(status.p, 0, sizeof(int), s));
  double* dev = dev_in ? (double*)ds.dptr : nullptr;
  double* nul = null_in ? (double*)ns.dptr : nullptr;
  if (!dev) {
    tdev.alloc(r, s);
    dev = tdev.p;
  }
  if (!nul) {
    tnull.alloc(r, s);
    nul = tnull.p;
  }
  const int ne = k * kb;
  auto cross_of = [&](const double* Wm) {
    {
      KScope ks_("k_glm_cross", s, 8.0 * (double)n * kb);
      k_glm_cross<<<nblk, GT, 0, s>>>(Z, ldz, n, k, Wm, Y, ldy, r, part.p);
    }
    {
      KScope ks_("k_reduce_partials", s, 0.0);
      k_reduce_partials<<<(unsigned)ceil_div(ne, 128), 128, 0, s>>>(part.p, nblk, ne, cross.p);
    }
  };
  cross_of(nullptr);  // Z^T [Z | Y]
  {
    KScope ks_("k_glm_chol", s, 0.0);
    k_glm_chol<<<1, 128, 0, s>>>(cross.p, k, nullptr, W1.p, status.p);
  }
  cross_of(W1.p);  // (Z W1)^T [Z W1 | Y]
  {
    KScope ks_("k_glm_chol", s, 0.0);
    k_glm_chol<<<1, 128, 0, s>>>(cross.p, k, W1.p, W.p, status.p);
  }
  cross_of(W.p);  // Q^T Y in columns k..
  {
    KScope ks_("k_glm_coef", s, 0.0);
    k_glm_coef<<<(unsigned)ceil_div(k * r, 128), 128, 0, s>>>(cross.p, W.p, k, r, (double*)cs.dptr);
  }
  for (int pass = 0; pass < 2; ++pass) {
    {
      KScope ks_("k_glm_dev", s, 8.0 * (double)n * (r + (pass ? k : 0)));
      k_glm_dev<<<nblk, GT, 0, s>>>(Z, ldz, n, k, Y, ldy, r, (const double*)cs.dptr, mean.p, pass, dpart.p);
    }
    {
      KScope ks_("k_glm_dev_final", s, 0.0);
      k_glm_dev_final<<<(unsigned)ceil_div(r, 64), 64, 0, s>>>(dpart.p, nblk, r, n, pass, mean.p, dev, nul);
    }
  }
  BF_CUDA_CHECK(cudaGetLastError());
  int hs = 0;
  BF_CUDA_CHECK(cudaMemcpyAsync(&hs, status.p, sizeof(int), cudaMemcpyDeviceToHost, s));
  cs.finish(s);
  if (dev_in) ds.finish(s);
  if (null_in) ns.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_REQUIRE(hs == 0, BF_EINVAL, "bf_glm_gaussian: design matrix is rank deficient");
}

void rank_similarity_impl(const double* a_in, const double* b_in, int32_t p, double* out_in, cudaStream_t s) {
  InStage as(a_in, sizeof(double) * (size_t)p, s), bs(b_in, sizeof(double) * (size_t)p, s);
  OutStage os(out_in, sizeof(double) * 2, s);
  const size_t smem = sizeof(double) * 2 * (size_t)p;
  static int smax = 0;
  if (!smax) smax = dyn_smem_limit(k_rank_similarity);
  BF_REQUIRE(smem <= (size_t)smax, BF_EINVAL, "bf_rank_similarity: p too large for shared memory");
  {
    KScope ks_("k_rank_similarity", s, 0.0);
    k_rank_similarity<<<1, RT, smem, s>>>((const double*)as.dptr, (const double*)bs.dptr, p, (double*)os.dptr);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  os.finish(s);
  if (os.host || as.tmp.p || bs.tmp.p) BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

}  // namespace bf
