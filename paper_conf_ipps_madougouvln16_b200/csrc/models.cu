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
#include <vector>


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

// ------------------------------------------------------------------ MARS (reading R28)
// Forward pass: every candidate (v, t) is one CTA that sums, over the rows, the products of its two hinges
// c1 = max(0, x_v - t), c2 = max(0, t - x_v) with the orthonormal basis Q (16 columns per pass), with
// themselves and with the residual r (fixed-order block reductions).  The RSS of basis + pair is
// RSS - b^T G^-1 b with G = [c_i.c_j - (Q^T c_i).(Q^T c_j)] (c1.c2 = 0: disjoint supports), b = [c_i.r];
// a column whose projected norm is below 1e-10 of its norm lies in span(Q) and is left out (the oracle's
// rank-deficient least squares).  The accepted pair is appended to B and, orthogonalised twice (CGS2), to Q.
constexpr int MQC = 16;  // Q columns per candidate pass
constexpr int MNT = 256;

__device__ __forceinline__ double block_sum_d(double v, double* red) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
  __syncthreads();
  if (lane == 0) red[wid] = v;
  __syncthreads();
  double t = 0.0;
  for (int w = 0; w < MNT / 32; ++w) t += red[w];
  return t;
}

// sums[c * SW + ...]: [0, 2M) = Q^T c1, Q^T c2 interleaved per column; 2M.. = c1.c1, c2.c2, c1.r, c2.r
__global__ void __launch_bounds__(MNT) k_mars_cand(const double* __restrict__ X, int64_t ldx, int64_t n,
                                                  const int32_t* __restrict__ cvar, const double* __restrict__ cknot,
                                                  const double* __restrict__ Q, int M, const double* __restrict__ r,
                                                  int SW, double* __restrict__ sums) {
  __shared__ double red[MNT / 32];
  const int c = blockIdx.x;
  const int v = cvar[c];
  const double t = cknot[c];
  const double* x = X + (int64_t)v * ldx;
  double* out = sums + (int64_t)c * SW;
  for (int j0 = 0; j0 < M; j0 += MQC) {
    double a1[MQC], a2[MQC];
#pragma unroll
    for (int u = 0; u < MQC; ++u) a1[u] = a2[u] = 0.0;
    for (int64_t i = threadIdx.x; i < n; i += MNT) {
      const double xi = x[i], h1 = fmax(xi - t, 0.0), h2 = fmax(t - xi, 0.0);
#pragma unroll
      for (int u = 0; u < MQC; ++u)
        if (j0 + u < M) {
          const double q = Q[(int64_t)(j0 + u) * n + i];
          a1[u] += h1 * q;
          a2[u] += h2 * q;
        }
    }
    for (int u = 0; u < MQC && j0 + u < M; ++u) {
      const double s1 = block_sum_d(a1[u], red), s2 = block_sum_d(a2[u], red);
      if (threadIdx.x == 0) {
        out[2 * (j0 + u)] = s1;
        out[2 * (j0 + u) + 1] = s2;
      }
    }
  }
  double e11 = 0.0, e22 = 0.0, e1r = 0.0, e2r = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += MNT) {
    const double xi = x[i], h1 = fmax(xi - t, 0.0), h2 = fmax(t - xi, 0.0), ri = r[i];
    e11 += h1 * h1;
    e22 += h2 * h2;
    e1r += h1 * ri;
    e2r += h2 * ri;
  }
  e11 = block_sum_d(e11, red);
  e22 = block_sum_d(e22, red);
  e1r = block_sum_d(e1r, red);
  e2r = block_sum_d(e2r, red);
  if (threadIdx.x == 0) {
    out[2 * M] = e11;
    out[2 * M + 1] = e22;
    out[2 * M + 2] = e1r;
    out[2 * M + 3] = e2r;
  }
}

// RSS of basis + pair for every candidate; then (one CTA) the chosen candidate by R28's tie rule:
// the lowest index among those within tol * TSS of the minimum (candidates are in (v, t) order).
__global__ void k_mars_rss(const double* __restrict__ sums, int SW, int M, int K, double rss0,
                           double* __restrict__ rss) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= K) return;
  const double* s = sums + (int64_t)c * SW;
  double g11 = s[2 * M], g22 = s[2 * M + 1], g12 = 0.0;
  const double n11 = g11, n22 = g22;
  for (int j = 0; j < M; ++j) {
    g11 -= s[2 * j] * s[2 * j];
    g22 -= s[2 * j + 1] * s[2 * j + 1];
    g12 -= s[2 * j] * s[2 * j + 1];
  }
  const double b1 = s[2 * M + 2], b2 = s[2 * M + 3];
  const bool ok1 = g11 > 1e-10 * n11 && n11 > 0.0, ok2 = g22 > 1e-10 * n22 && n22 > 0.0;
  double drop = 0.0;
  if (ok1 && ok2) {
    const double det = g11 * g22 - g12 * g12;
    drop = det > 1e-12 * g11 * g22 ? (g22 * b1 * b1 - 2.0 * g12 * b1 * b2 + g11 * b2 * b2) / det
                                   : fmax(b1 * b1 / g11, b2 * b2 / g22);
  } else if (ok1) {
    drop = b1 * b1 / g11;
  } else if (ok2) {
    drop = b2 * b2 / g22;
  }
  rss[c] = fmax(rss0 - drop, 0.0);
}

__global__ void k_mars_pick(const double* __restrict__ rss, int K, double tolabs, int* __restrict__ pick,
                            double* __restrict__ prss) {
  __shared__ double sm[MNT];
  __shared__ int si[MNT];
  double m = 1e308;
  for (int c = threadIdx.x; c < K; c += MNT) m = fmin(m, rss[c]);
  sm[threadIdx.x] = m;
  __syncthreads();
  for (int s = MNT / 2; s > 0; s >>= 1) {
    if (threadIdx.x < s) sm[threadIdx.x] = fmin(sm[threadIdx.x], sm[threadIdx.x + s]);
    __syncthreads();
  }
  const double lim = sm[0] + tolabs;
  __syncthreads();
  int best = K;
  for (int c = threadIdx.x; c < K; c += MNT)
    if (rss[c] <= lim) {
      best = c;
      break;
    }
  si[threadIdx.x] = best;
  __syncthreads();
  for (int s = MNT / 2; s > 0; s >>= 1) {
    if (threadIdx.x < s) si[threadIdx.x] = min(si[threadIdx.x], si[threadIdx.x + s]);
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    *pick = si[0] < K ? si[0] : -1;
    *prss = si[0] < K ? rss[si[0]] : 0.0;
  }
}

// Append column `col` (hinge of candidate c, direction dir; dir 0 = the intercept) to B, and to Q after two
// Gram-Schmidt passes unless it lies in span(Q); then r -= q (q . r).  One CTA (n is the counter-model size).
__global__ void __launch_bounds__(MNT) k_mars_append(const double* __restrict__ X, int64_t ldx, int64_t n, int v,
                                                    double t, int dir, double* __restrict__ B, int mb,
                                                    double* __restrict__ Q, int* __restrict__ Mq, double* __restrict__ r,
                                                    double* __restrict__ w) {
  __shared__ double red[MNT / 32];
  __shared__ double dots[GMAXK];
  const double* x = X + (int64_t)v * ldx;
  const int M = *Mq;
  double nn = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += MNT) {
    const double h = dir == 0 ? 1.0 : dir > 0 ? fmax(x[i] - t, 0.0) : fmax(t - x[i], 0.0);
    B[(int64_t)mb * n + i] = h;
    w[i] = h;
    nn += h * h;
  }
  nn = block_sum_d(nn, red);
  for (int pass = 0; pass < 2; ++pass) {
    for (int j = 0; j < M; ++j) {
      double s = 0.0;
      for (int64_t i = threadIdx.x; i < n; i += MNT) s += Q[(int64_t)j * n + i] * w[i];
      s = block_sum_d(s, red);
      if (threadIdx.x == 0) dots[j] = s;
    }
    __syncthreads();
    for (int64_t i = threadIdx.x; i < n; i += MNT) {
      double wi = w[i];
      for (int j = 0; j < M; ++j) wi -= dots[j] * Q[(int64_t)j * n + i];
      w[i] = wi;
    }
    __syncthreads();
  }
  double qq = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += MNT) qq += w[i] * w[i];
  qq = block_sum_d(qq, red);
  if (!(qq > 1e-20 * nn) || nn == 0.0) return;  // in span(Q): B keeps the column, Q does not grow
  const double inv = 1.0 / sqrt(qq);
  double qr = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += MNT) {
    const double q = w[i] * inv;
    Q[(int64_t)M * n + i] = q;
    qr += q * r[i];
  }
  qr = block_sum_d(qr, red);
  for (int64_t i = threadIdx.x; i < n; i += MNT) r[i] -= Q[(int64_t)M * n + i] * qr;
  __syncthreads();
  if (threadIdx.x == 0) *Mq = M + 1;
}

__global__ void k_mars_rss_direct(const double* __restrict__ r, int64_t n, double* __restrict__ out) {
  __shared__ double red[MNT / 32];
  double s = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += MNT) s += r[i] * r[i];
  s = block_sum_d(s, red);
  if (threadIdx.x == 0) *out = s;
}

// Backward pass (one CTA).  With the forward pass's orthonormal Q (Mq columns) and R = Q^T B, d = Q^T y,
// RSS(S) = RSS_perp + min_c || d - R_S c ||^2 (B = Q R, y = Q d + r_perp), a least-squares problem of at most
// 32 x 31 solved by Householder QR with column skipping (a column whose remaining norm is below 1e-12 of its
// norm is dependent: the rank-deficient least squares of the oracle).  No normal equations: the RSS of
// nearly dependent subsets (hinge pairs at close knots) stays accurate, so R28's tie rules decide the same
// way as the oracle's lstsq.  Each step, thread j evaluates the removal of term j (its own local scratch).
__device__ double qr_subset_rss(const double* Rm, const double* dv, int Mq, int M, unsigned mask, double* A, double* b,
                                double* coef) {
  int cols[GMAXK], k = 0;
  for (int j = 0; j < M; ++j)
    if ((mask >> j) & 1u) cols[k++] = j;
  for (int c = 0; c < k; ++c)
    for (int i = 0; i < Mq; ++i) A[c * GMAXK + i] = Rm[(int64_t)cols[c] * Mq + i];
  for (int i = 0; i < Mq; ++i) b[i] = dv[i];
  int r = 0;
  int piv[GMAXK];
  for (int c = 0; c < k; ++c) {
    double cn = 0.0, nr = 0.0;
    for (int i = 0; i < Mq; ++i) cn += A[c * GMAXK + i] * A[c * GMAXK + i];
    for (int i = r; i < Mq; ++i) nr += A[c * GMAXK + i] * A[c * GMAXK + i];
    piv[c] = -1;
    if (r >= Mq || !(nr > 1e-24 * cn) || cn == 0.0) continue;  // dependent column
    const double alpha = A[c * GMAXK + r] > 0.0 ? -sqrt(nr) : sqrt(nr);
    const double v0 = A[c * GMAXK + r] - alpha;
    const double vnorm2 = nr - A[c * GMAXK + r] * A[c * GMAXK + r] + v0 * v0;
    // reflect columns c.. and b with v = (v0, A[r+1.., c])
    for (int c2 = c; c2 < k; ++c2) {
      double t = v0 * A[c2 * GMAXK + r];
      for (int i = r + 1; i < Mq; ++i) t += A[c * GMAXK + i] * A[c2 * GMAXK + i];
      if (c2 == c) continue;
      t = 2.0 * t / vnorm2;
      A[c2 * GMAXK + r] -= t * v0;
      for (int i = r + 1; i < Mq; ++i) A[c2 * GMAXK + i] -= t * A[c * GMAXK + i];
    }
    {
      double t = v0 * b[r];
      for (int i = r + 1; i < Mq; ++i) t += A[c * GMAXK + i] * b[i];
      t = 2.0 * t / vnorm2;
      b[r] -= t * v0;
      for (int i = r + 1; i < Mq; ++i) b[i] -= t * A[c * GMAXK + i];
    }
    A[c * GMAXK + r] = alpha;
    piv[c] = r;
    ++r;
  }
  double res = 0.0;
  for (int i = r; i < Mq; ++i) res += b[i] * b[i];
  if (coef) {  // back substitution over the kept columns (rows piv[c]); dependent columns get 0
    for (int c = 0; c < k; ++c) coef[cols[c]] = 0.0;
    for (int c = k - 1; c >= 0; --c) {
      if (piv[c] < 0) continue;
      const int rr = piv[c];
      double t = b[rr];
      for (int c2 = c + 1; c2 < k; ++c2)
        if (piv[c2] >= 0) t -= A[c2 * GMAXK + rr] * coef[cols[c2]];
      coef[cols[c]] = t / A[c * GMAXK + rr];
    }
  }
  return res;
}

// qty: Q^T [B | y] as an Mq x (M + 1) column-major block (column M = Q^T y); rss_perp = || y - Q Q^T y ||^2.
__global__ void k_mars_backward(const double* __restrict__ qty, int Mq, int M, double rss_perp, double tss, int64_t n,
                                double penalty, double* __restrict__ scratch, unsigned* __restrict__ best_mask,
                                double* __restrict__ coef) {
  __shared__ double rj[GMAXK];
  __shared__ unsigned sS, sbest;
  __shared__ double sbg;
  const int tid = threadIdx.x;
  const double tol = 1e-12 * tss;
  const double* Rm = qty;
  const double* dv = qty + (int64_t)M * Mq;
  auto gcv = [&](double rr, int m) {
    const double C = m + penalty * (m - 1) / 2.0;
    const double dd = 1.0 - C / (double)n;
    return (rr / (double)n) / (dd * dd);
  };
  // per thread (global, L1-cached): GMAXK * GMAXK (A) + GMAXK (b)
  double* myA = scratch + (size_t)tid * (GMAXK * GMAXK + GMAXK);
  double* myb = myA + GMAXK * GMAXK;
  if (tid == 0) {
    sS = (M >= 32) ? 0xffffffffu : ((1u << M) - 1u);
    sbest = sS;
    sbg = gcv(rss_perp + qr_subset_rss(Rm, dv, Mq, M, sS, myA, myb, nullptr), M);
  }
  __syncthreads();
  for (int m = M; m > 1; --m) {
    const unsigned S = sS;
    if (tid >= 1 && tid < M && ((S >> tid) & 1u)) rj[tid] = rss_perp + qr_subset_rss(Rm, dv, Mq, M, S & ~(1u << tid), myA, myb, nullptr);
    __syncthreads();
    if (tid == 0) {
      double rmin = 1e308;
      for (int j = 1; j < M; ++j)
        if ((S >> j) & 1u) rmin = fmin(rmin, rj[j]);
      int drop = -1;
      for (int j = 1; j < M && drop < 0; ++j)
        if (((S >> j) & 1u) && rj[j] <= rmin + tol) drop = j;
      sS = S & ~(1u << drop);
      const double g = gcv(rj[drop], m - 1);
      if (g <= sbg + tol / (double)n) {
        sbg = g;
        sbest = sS;
      }
    }
    __syncthreads();
  }
  if (tid == 0) {
    double cf[GMAXK];
    qr_subset_rss(Rm, dv, Mq, M, sbest, myA, myb, cf);
    *best_mask = sbest;
    for (int j = 0; j < M; ++j) coef[j] = ((sbest >> j) & 1u) ? cf[j] : 0.0;
  }
}

// residual of the chosen model (for its RSS), and the model on new rows
__global__ void k_mars_eval(const double* __restrict__ X, int64_t ldx, int64_t n, int nt, const int32_t* __restrict__ tv,
                            const double* __restrict__ tk, const int32_t* __restrict__ td, const double* __restrict__ coef,
                            const double* __restrict__ y, double* __restrict__ out) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  double f = 0.0;
  for (int j = 0; j < nt; ++j) {
    const int d = td[j];
    const double h = d == 0 ? 1.0 : d > 0 ? fmax(X[(int64_t)tv[j] * ldx + i] - tk[j], 0.0)
                                          : fmax(tk[j] - X[(int64_t)tv[j] * ldx + i], 0.0);
    f += coef[j] * h;
  }
  out[i] = y ? y[i] - f : f;
}

// order-preserving 64-bit key of the canonical value (-0 -> +0, R18) for the hand-written radix sort, and back
__global__ void k_mars_key(const double* __restrict__ x, int64_t n, uint64_t* __restrict__ out) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint64_t b = (uint64_t)__double_as_longlong(__dadd_rn(x[i], 0.0));
  out[i] = (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}
__global__ void k_mars_unkey(const uint64_t* __restrict__ k, int64_t n, double* __restrict__ out) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint64_t v = k[i];
  out[i] = __longlong_as_double((long long)((v >> 63) ? (v & 0x7fffffffffffffffull) : ~v));
}
__global__ void k_mars_sums(const double* __restrict__ y, int64_t n, double* __restrict__ out /* tss, yy */) {
  __shared__ double red[MNT / 32];
  double s = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += MNT) s += y[i];
  s = block_sum_d(s, red);
  const double mean = s / (double)n;
  double t = 0.0, q = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += MNT) {
    const double dv = y[i] - mean;
    t += dv * dv;
    q += y[i] * y[i];
  }
  t = block_sum_d(t, red);
  q = block_sum_d(q, red);
  if (threadIdx.x == 0) {
    out[0] = t;
    out[1] = q;
  }
}

}  // namespace

void mars_fit_impl(const double* X_in, int64_t ldx, int64_t n, int32_t d, const double* y_in, int32_t nk, double thresh,
                   double penalty, int32_t* nterms, int32_t* tvar, double* tknot, int32_t* tdir, double* coef_out,
                   double* stats, cudaStream_t s) {
  if (nk <= 0) nk = std::min(200, std::max(20, 2 * d)) + 1;
  BF_REQUIRE(d >= 1 && nk >= 1 && nk <= GMAXK - 1 && n >= 2, BF_EINVAL,
             "bf_mars_fit: need d >= 1, n >= 2 and at most 31 terms (d <= 15 with the default nk)");
  InStage Xs(X_in, sizeof(double) * (size_t)(ldx * (d - 1) + n), s), ys(y_in, sizeof(double) * (size_t)n, s);
  const double* X = (const double*)Xs.dptr;
  const double* y = (const double*)ys.dptr;
  // candidate knots: the distinct values of every predictor other than its minimum and maximum
  std::vector<int32_t> hv;
  std::vector<double> hk;
  {
    DBuf<uint64_t> k0(n, s), k1(n, s), uk(n, s);
    DBuf<double> uq(n, s);
    DBuf<int32_t> nu(1, s);
    std::vector<double> hu;
    for (int v = 0; v < d; ++v) {
      k_mars_key<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>(X + (int64_t)v * ldx, n, k0.p);
      const uint64_t* srt = radix_sort_u64(k0.p, k1.p, nullptr, nullptr, n, 1, s, nullptr);
      unique_u64(srt, n, uk.p, nu.p, s);
      k_mars_unkey<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>(uk.p, n, uq.p);
      BF_CUDA_CHECK(cudaGetLastError());
      int hn = 0;
      BF_CUDA_CHECK(cudaMemcpyAsync(&hn, nu.p, sizeof(int), cudaMemcpyDeviceToHost, s));
      BF_CUDA_CHECK(cudaStreamSynchronize(s));
      if (hn > 2) {
        hu.resize(hn);
        BF_CUDA_CHECK(cudaMemcpyAsync(hu.data(), uq.p, sizeof(double) * hn, cudaMemcpyDeviceToHost, s));
        BF_CUDA_CHECK(cudaStreamSynchronize(s));
        for (int k = 1; k + 1 < hn; ++k) {
          hv.push_back(v);
          hk.push_back(hu[k]);
        }
      }
    }
  }
  const int K = (int)hv.size();
  DBuf<int32_t> cvar(std::max(K, 1), s);
  DBuf<double> cknot(std::max(K, 1), s);
  if (K) {
    BF_CUDA_CHECK(cudaMemcpyAsync(cvar.p, hv.data(), sizeof(int32_t) * K, cudaMemcpyHostToDevice, s));
    BF_CUDA_CHECK(cudaMemcpyAsync(cknot.p, hk.data(), sizeof(double) * K, cudaMemcpyHostToDevice, s));
  }
  const int SW = 2 * nk + 4;
  DBuf<double> B((size_t)n * (nk + 1), s), Q((size_t)n * nk, s), r(n, s), w(n, s), sums((size_t)std::max(K, 1) * SW, s),
      crss(std::max(K, 1), s), sc(4, s), prss(1, s);
  DBuf<int> Mq(1, s), pick(1, s);
  const int* Mq_dev_ptr = Mq.p;
  BF_CUDA_CHECK(cudaMemsetAsync(Mq.p, 0, sizeof(int), s));
  BF_CUDA_CHECK(cudaMemcpyAsync(r.p, y, sizeof(double) * n, cudaMemcpyDeviceToDevice, s));
  double hs[2];
  {
    KScope ks_("k_mars_sums", s, 0.0);
    k_mars_sums<<<1, MNT, 0, s>>>(y, n, sc.p);
  }
  BF_CUDA_CHECK(cudaMemcpyAsync(hs, sc.p, sizeof(double) * 2, cudaMemcpyDeviceToHost, s));
  auto append = [&](int v, double t, int dir, int mb) {
    KScope ks_("k_mars_append", s, 0.0);
    k_mars_append<<<1, MNT, 0, s>>>(X, ldx, n, v, t, dir, B.p, mb, Q.p, Mq.p, r.p, w.p);
  };
  auto rss_now = [&]() {
    double h = 0.0;
    k_mars_rss_direct<<<1, MNT, 0, s>>>(r.p, n, prss.p);
    BF_CUDA_CHECK(cudaMemcpyAsync(&h, prss.p, sizeof(double), cudaMemcpyDeviceToHost, s));
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
    return h;
  };
  append(0, 0.0, 0, 0);  // intercept
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  const double tss = hs[0];
  double rss = rss_now();
  std::vector<int32_t> fv{0};
  std::vector<double> fk{0.0};
  std::vector<int32_t> fd{0};
  int M = 1;
  while (M + 2 <= nk && tss > 0.0 && K > 0) {
    int hq = 0;
    BF_CUDA_CHECK(cudaMemcpyAsync(&hq, Mq.p, sizeof(int), cudaMemcpyDeviceToHost, s));
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
    {
      KScope ks_("k_mars_cand", s, 8.0 * (double)K * n * (hq + 2));
      k_mars_cand<<<K, MNT, 0, s>>>(X, ldx, n, cvar.p, cknot.p, Q.p, hq, r.p, SW, sums.p);
    }
    {
      KScope ks_("k_mars_rss", s, 0.0);
      k_mars_rss<<<(unsigned)ceil_div(K, 128), 128, 0, s>>>(sums.p, SW, hq, K, rss, crss.p);
    }
    {
      KScope ks_("k_mars_pick", s, 0.0);
      k_mars_pick<<<1, MNT, 0, s>>>(crss.p, K, 1e-12 * tss, pick.p, prss.p);
    }
    BF_CUDA_CHECK(cudaGetLastError());
    int hp = -1;
    double hr = 0.0;
    BF_CUDA_CHECK(cudaMemcpyAsync(&hp, pick.p, sizeof(int), cudaMemcpyDeviceToHost, s));
    BF_CUDA_CHECK(cudaMemcpyAsync(&hr, prss.p, sizeof(double), cudaMemcpyDeviceToHost, s));
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
    if (hp < 0 || (rss - hr) / tss < thresh) break;
    append(hv[hp], hk[hp], 1, M);
    append(hv[hp], hk[hp], -1, M + 1);
    fv.insert(fv.end(), {hv[hp], hv[hp]});
    fk.insert(fk.end(), {hk[hp], hk[hp]});
    fd.insert(fd.end(), {1, -1});
    M += 2;
    rss = rss_now();
    if (1.0 - rss / tss >= 1.0 - thresh) break;
  }
  // backward pass on R = Q^T B, d = Q^T y (k_glm_cross: Q^T [Q | B | y]; Q has Mq <= M columns)
  int nq = 0;
  BF_CUDA_CHECK(cudaMemcpyAsync(&nq, Mq_dev_ptr, sizeof(int), cudaMemcpyDeviceToHost, s));
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_CUDA_CHECK(cudaMemcpyAsync(B.p + (size_t)M * n, y, sizeof(double) * n, cudaMemcpyDeviceToDevice, s));
  const int nblk = (int)std::max<int64_t>(1, std::min<int64_t>(296, ceil_div(n, GROWS)));
  const int ne = nq * (nq + M + 1);
  DBuf<double> part((size_t)nblk * ne, s), cross(ne, s), cf(M, s), bscr((size_t)32 * (GMAXK * GMAXK + GMAXK), s);
  DBuf<unsigned> bm(1, s);
  {
    KScope ks_("k_glm_cross", s, 8.0 * (double)n * (nq + M + 1));
    k_glm_cross<<<nblk, GT, 0, s>>>(Q.p, n, n, nq, nullptr, B.p, n, M + 1, part.p);
  }
  k_reduce_partials<<<(unsigned)ceil_div(ne, 128), 128, 0, s>>>(part.p, nblk, ne, cross.p);
  {
    KScope ks_("k_mars_backward", s, 0.0);
    k_mars_backward<<<1, 32, 0, s>>>(cross.p + (size_t)nq * nq, nq, M, rss, tss, n, penalty, bscr.p, bm.p, cf.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  unsigned hb = 0;
  std::vector<double> hc(M);
  BF_CUDA_CHECK(cudaMemcpyAsync(&hb, bm.p, sizeof(unsigned), cudaMemcpyDeviceToHost, s));
  BF_CUDA_CHECK(cudaMemcpyAsync(hc.data(), cf.p, sizeof(double) * M, cudaMemcpyDeviceToHost, s));
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  int nt = 0;
  for (int j = 0; j < M; ++j)
    if ((hb >> j) & 1u) {
      tvar[nt] = fv[j];
      tknot[nt] = fk[j];
      tdir[nt] = fd[j];
      coef_out[nt] = hc[j];
      ++nt;
    }
  *nterms = nt;
  // RSS of the chosen model from its residual; GCV and RSq (R28)
  DBuf<int32_t> dv(nt, s), dd(nt, s);
  DBuf<double> dk(nt, s), dc(nt, s);
  BF_CUDA_CHECK(cudaMemcpyAsync(dv.p, tvar, sizeof(int32_t) * nt, cudaMemcpyHostToDevice, s));
  BF_CUDA_CHECK(cudaMemcpyAsync(dd.p, tdir, sizeof(int32_t) * nt, cudaMemcpyHostToDevice, s));
  BF_CUDA_CHECK(cudaMemcpyAsync(dk.p, tknot, sizeof(double) * nt, cudaMemcpyHostToDevice, s));
  BF_CUDA_CHECK(cudaMemcpyAsync(dc.p, coef_out, sizeof(double) * nt, cudaMemcpyHostToDevice, s));
  {
    KScope ks_("k_mars_eval", s, 8.0 * (double)n * (nt + 2));
    k_mars_eval<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>(X, ldx, n, nt, dv.p, dk.p, dd.p, dc.p, y, r.p);
  }
  const double rb = rss_now();
  const double C = nt + penalty * (nt - 1) / 2.0, den = 1.0 - C / (double)n;
  stats[0] = rb;
  stats[1] = (rb / (double)n) / (den * den);
  stats[2] = tss > 0.0 ? 1.0 - rb / tss : 1.0;
}

void mars_predict_impl(const double* X_in, int64_t ldx, int64_t m, int32_t d, int32_t nt, const int32_t* tvar,
                       const double* tknot, const int32_t* tdir, const double* coef, double* out_in, cudaStream_t s) {
  if (m == 0 || nt == 0) return;
  InStage Xs(X_in, sizeof(double) * (size_t)(ldx * (d - 1) + m), s);
  OutStage os(out_in, sizeof(double) * (size_t)m, s);
  DBuf<int32_t> dv(nt, s), dd(nt, s);
  DBuf<double> dk(nt, s), dc(nt, s);
  BF_CUDA_CHECK(cudaMemcpyAsync(dv.p, tvar, sizeof(int32_t) * nt, cudaMemcpyDefault, s));
  BF_CUDA_CHECK(cudaMemcpyAsync(dd.p, tdir, sizeof(int32_t) * nt, cudaMemcpyDefault, s));
  BF_CUDA_CHECK(cudaMemcpyAsync(dk.p, tknot, sizeof(double) * nt, cudaMemcpyDefault, s));
  BF_CUDA_CHECK(cudaMemcpyAsync(dc.p, coef, sizeof(double) * nt, cudaMemcpyDefault, s));
  {
    KScope ks_("k_mars_eval", s, 8.0 * (double)m * (nt + 1));
    k_mars_eval<<<(unsigned)ceil_div(m, 256), 256, 0, s>>>((const double*)Xs.dptr, ldx, m, nt, dv.p, dk.p, dd.p, dc.p,
                                                         nullptr, (double*)os.dptr);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  os.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

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

// ------------------------------------------------------------------ workflow statistics (NEXT-3 / NEXT-4)
namespace bf {
namespace {
constexpr int WNT = 256;
__device__ double wf_block_sum(double v, double* red) {
  for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;
  __syncthreads();
  double t = 0.0;
  if (threadIdx.x == 0)
    for (int k = 0; k < WNT / 32; ++k) t += red[k];
  __syncthreads();
  return t;  // valid in thread 0
}
// Reading R26's default design: u = (log2 s - mean) / sd (sample sd, n - 1), rows [1, u, u^2, u^3].  One CTA
// computes the statistics in a fixed order; the rows are written by a grid.
__global__ void k_log_stats(const double* s, int64_t n, double* st /* mean, sd */) {
  __shared__ double red[WNT / 32];
  __shared__ double s_mean;
  double a = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += WNT) a += log2(s[i]);
  a = wf_block_sum(a, red);
  if (threadIdx.x == 0) s_mean = a / (double)n;
  __syncthreads();
  const double mean = s_mean;
  double v = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += WNT) {
    const double d = log2(s[i]) - mean;
    v += d * d;
  }
  v = wf_block_sum(v, red);
  if (threadIdx.x == 0) {
    st[0] = mean;
    st[1] = n > 1 ? sqrt(v / (double)(n - 1)) : 0.0;
  }
}
__global__ void k_log_design(const double* s, int64_t n, const double* st, double* Z, int64_t ldz) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  const double u = (log2(s[i]) - st[0]) / st[1];
  Z[i] = 1.0;
  Z[ldz + i] = u;
  Z[2 * ldz + i] = u * u;
  Z[3 * ldz + i] = u * u * u;
}
// Test error of predicted times ("variance explained"): mse = mean (yhat - y)^2,
// explained = 1 - mse / mean (y - mean y)^2 (NaN for constant y).
__global__ void k_pred_error(const double* yh, const double* y, int64_t m, double* out) {
  __shared__ double red[WNT / 32];
  __shared__ double s_mean;
  double a = 0.0, e = 0.0;
  for (int64_t i = threadIdx.x; i < m; i += WNT) {
    a += y[i];
    const double d = yh[i] - y[i];
    e += d * d;
  }
  a = wf_block_sum(a, red);
  e = wf_block_sum(e, red);
  if (threadIdx.x == 0) s_mean = a / (double)m;
  __syncthreads();
  const double mean = s_mean;
  double v = 0.0;
  for (int64_t i = threadIdx.x; i < m; i += WNT) {
    const double d = y[i] - mean;
    v += d * d;
  }
  v = wf_block_sum(v, red);
  if (threadIdx.x == 0) {
    const double mse = e / (double)m, var = v / (double)m;
    out[0] = mse;
    out[1] = var > 0.0 ? 1.0 - mse / var : __longlong_as_double(0x7ff8000000000000ll);
  }
}
}  // namespace

void log_size_design_impl(const double* s_in, int64_t n, double* Z_in, int64_t ldz, cudaStream_t s) {
  InStage ss(s_in, sizeof(double) * (size_t)n, s);
  OutStage zs(Z_in, sizeof(double) * (size_t)(3 * ldz + n), s);
  DBuf<double> st(2, s);
  {
    KScope ks_("k_log_design", s, 0.0, 2);
    k_log_stats<<<1, WNT, 0, s>>>((const double*)ss.dptr, n, st.p);
    k_log_design<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>((const double*)ss.dptr, n, st.p, (double*)zs.dptr, ldz);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  zs.finish(s);
  if (zs.host || ss.tmp.p) BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

void prediction_error_impl(const double* yh_in, const double* y_in, int64_t m, double* out_host, cudaStream_t s) {
  InStage a(yh_in, sizeof(double) * (size_t)m, s), b(y_in, sizeof(double) * (size_t)m, s);
  DBuf<double> o(2, s);
  {
    KScope ks_("k_pred_error", s, 16.0 * (double)m);
    k_pred_error<<<1, WNT, 0, s>>>((const double*)a.dptr, (const double*)b.dptr, m, o.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  BF_CUDA_CHECK(cudaMemcpyAsync(out_host, o.p, 2 * sizeof(double), cudaMemcpyDeviceToHost, s));
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
}
}  // namespace bf
