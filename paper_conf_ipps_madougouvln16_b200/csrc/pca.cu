// pca.cu -- counter PCA (P:134, P:177 prcomp; S9).
//
//   k_colstats : column means and (if scale) sample standard deviations, fp64.
//   k_gram     : Z^T Z over row tiles staged in shared memory; each CTA keeps
//                its own partial Gram (one owner thread per (i, j>=i) entry),
//                partials are summed in fixed order -> deterministic C.
//   k_jacobi   : one CTA, C and V resident in shared memory, parallel cyclic
//                Jacobi with round-robin (tournament) pairing: p/2 disjoint
//                rotations per round.
//   k_scores   : scores = Z V[:, :k].
// The Gram is a p x p fp64 contraction of n rows (AI ~ p/4 flop/B); it runs in
// microseconds at the config sizes, so it stays on the fp64 CUDA cores.
#include <algorithm>
#include <cmath>

#include "bf_internal.cuh"

namespace bf {
namespace {

constexpr int NT = 256;
constexpr int GR = 32;  // rows per Gram tile

__global__ void k_colstats(const double* X, int64_t ldx, int64_t n, int scale, double* mu, double* sd) {
  __shared__ double sm[NT];
  const int j = blockIdx.x;
  const double* col = X + (int64_t)j * ldx;
  double s = 0.0;
  for (int64_t r = threadIdx.x; r < n; r += NT) s += col[r];
  sm[threadIdx.x] = s;
  __syncthreads();
  for (int o = NT / 2; o > 0; o >>= 1) {
    if (threadIdx.x < o) sm[threadIdx.x] += sm[threadIdx.x + o];
    __syncthreads();
  }
  const double m = sm[0] / (double)n;
  __syncthreads();
  double v = 0.0;
  if (scale)
    for (int64_t r = threadIdx.x; r < n; r += NT) {
      const double d = col[r] - m;
      v += d * d;
    }
  sm[threadIdx.x] = v;
  __syncthreads();
  for (int o = NT / 2; o > 0; o >>= 1) {
    if (threadIdx.x < o) sm[threadIdx.x] += sm[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    mu[j] = m;
    sd[j] = scale ? sqrt(sm[0] / (double)(n - 1)) : 1.0;
  }
}

__global__ void k_gram(const double* X, int64_t ldx, int64_t n, int p, const double* mu, const double* sd,
                       int scale, double* part) {
  extern __shared__ double sz[];  // GR x p tile, then npairs accumulators
  const int np = p * (p + 1) / 2;
  double* acc = sz + GR * p;
  for (int k = threadIdx.x; k < np; k += NT) acc[k] = 0.0;
  const int64_t ntile = (n + GR - 1) / GR;
  for (int64_t tile = blockIdx.x; tile < ntile; tile += gridDim.x) {
    const int64_t r0 = tile * GR;
    __syncthreads();
    for (int e = threadIdx.x; e < GR * p; e += NT) {
      const int j = e / GR, rr = e - j * GR;
      const int64_t r = r0 + rr;
      double z = 0.0;
      if (r < n) {
        z = X[(int64_t)j * ldx + r] - mu[j];
        if (scale) z = z / sd[j];
      }
      sz[rr * p + j] = z;
    }
    __syncthreads();
    for (int k = threadIdx.x; k < np; k += NT) {
      // pair index k -> (i, j), i <= j, row-major upper triangle
      int i = 0, rem = k;
      while (rem >= p - i) {
        rem -= p - i;
        ++i;
      }
      const int j = i + rem;
      double s = acc[k];
      for (int rr = 0; rr < GR; ++rr) s += sz[rr * p + i] * sz[rr * p + j];
      acc[k] = s;
    }
  }
  __syncthreads();
  for (int k = threadIdx.x; k < np; k += NT) part[(int64_t)blockIdx.x * np + k] = acc[k];
}

__global__ void k_gram_reduce(const double* part, int nparts, int p, int64_t n, double* C) {
  const int np = p * (p + 1) / 2;
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= np) return;
  double s = 0.0;
  for (int b = 0; b < nparts; ++b) s += part[(int64_t)b * np + k];
  int i = 0, rem = k;
  while (rem >= p - i) {
    rem -= p - i;
    ++i;
  }
  const int j = i + rem;
  const double c = s / (double)(n - 1);
  C[i * p + j] = c;
  C[j * p + i] = c;
}

// Parallel cyclic Jacobi on the symmetric p x p matrix (one CTA).
__global__ void k_jacobi(const double* Cin, int p, double* sdev, double* rot) {
  extern __shared__ double sm[];
  const int P = p + (p & 1);  // even number of players (a dummy if p is odd)
  double* A = sm;             // p x p
  double* V = A + p * p;      // p x p, column j = eigenvector j
  double* cs = V + p * p;     // P/2 x 2 (c, s)
  int* pi = (int*)(cs + P);   // P/2 x 2 (i, j)
  __shared__ double red[NT];
  __shared__ int s_stop;
  for (int e = threadIdx.x; e < p * p; e += NT) {
    A[e] = Cin[e];
    V[e] = (e / p == e % p) ? 1.0 : 0.0;
  }
  __syncthreads();
  double fro = 0.0;
  for (int e = threadIdx.x; e < p * p; e += NT) fro += A[e] * A[e];
  red[threadIdx.x] = fro;
  __syncthreads();
  for (int o = NT / 2; o > 0; o >>= 1) {
    if (threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
    __syncthreads();
  }
  const double fro2 = red[0];
  __syncthreads();
  for (int sweep = 0; sweep < 60; ++sweep) {
    // convergence: off(A)^2 <= (1e-15)^2 * ||A||_F^2
    double off = 0.0;
    for (int e = threadIdx.x; e < p * p; e += NT)
      if (e / p != e % p) off += A[e] * A[e];
    red[threadIdx.x] = off;
    __syncthreads();
    for (int o = NT / 2; o > 0; o >>= 1) {
      if (threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
      __syncthreads();
    }
    if (threadIdx.x == 0) s_stop = red[0] <= 1e-30 * fro2 || red[0] == 0.0;
    __syncthreads();
    if (s_stop) break;
    for (int round = 0; round < P - 1; ++round) {
      // circle method: player P-1 fixed, others rotate
      for (int k = threadIdx.x; k < P / 2; k += NT) {
        int i, j;
        if (k == 0) {
          i = P - 1;
          j = round;
        } else {
          i = (round + k) % (P - 1);
          j = (round - k + (P - 1)) % (P - 1);
        }
        if (i > j) {
          const int tmp = i;
          i = j;
          j = tmp;
        }
        double c = 1.0, s = 0.0;
        if (j < p) {
          const double aij = A[i * p + j];
          if (aij != 0.0) {
            const double th = (A[j * p + j] - A[i * p + i]) / (2.0 * aij);
            const double t = (th >= 0 ? 1.0 : -1.0) / (fabs(th) + sqrt(th * th + 1.0));
            c = 1.0 / sqrt(t * t + 1.0);
            s = t * c;
          }
        }
        pi[2 * k] = i;
        pi[2 * k + 1] = j;
        cs[2 * k] = c;
        cs[2 * k + 1] = s;
      }
      __syncthreads();
      // A <- A J ; V <- V J  (column rotations)
      for (int e = threadIdx.x; e < (P / 2) * p; e += NT) {
        const int k = e / p, r = e - k * p;
        const int i = pi[2 * k], j = pi[2 * k + 1];
        if (j >= p) continue;
        const double c = cs[2 * k], s = cs[2 * k + 1];
        const double ai = A[r * p + i], aj = A[r * p + j];
        A[r * p + i] = c * ai - s * aj;
        A[r * p + j] = s * ai + c * aj;
        const double vi = V[r * p + i], vj = V[r * p + j];
        V[r * p + i] = c * vi - s * vj;
        V[r * p + j] = s * vi + c * vj;
      }
      __syncthreads();
      // A <- J^T A (row rotations)
      for (int e = threadIdx.x; e < (P / 2) * p; e += NT) {
        const int k = e / p, r = e - k * p;
        const int i = pi[2 * k], j = pi[2 * k + 1];
        if (j >= p) continue;
        const double c = cs[2 * k], s = cs[2 * k + 1];
        const double ai = A[i * p + r], aj = A[j * p + r];
        A[i * p + r] = c * ai - s * aj;
        A[j * p + r] = s * ai + c * aj;
      }
      __syncthreads();
    }
  }
  // sort eigenvalues descending, sign rule, output
  if (threadIdx.x == 0) {
    int* order = pi;  // reuse (needs p ints; P/2*2 = P >= p)
    for (int j = 0; j < p; ++j) order[j] = j;
    for (int a = 0; a < p; ++a) {
      int best = a;
      for (int b = a + 1; b < p; ++b)
        if (A[order[b] * p + order[b]] > A[order[best] * p + order[best]]) best = b;
      const int tmp = order[a];
      order[a] = order[best];
      order[best] = tmp;
    }
  }
  __syncthreads();
  for (int jj = threadIdx.x; jj < p; jj += NT) {
    const int j = pi[jj];
    const double lam = A[j * p + j];
    sdev[jj] = sqrt(fmax(lam, 0.0));
    int im = 0;
    double vm = -1.0;
    for (int i = 0; i < p; ++i)
      if (fabs(V[i * p + j]) > vm) {
        vm = fabs(V[i * p + j]);
        im = i;
      }
    const double sg = V[im * p + j] < 0 ? -1.0 : 1.0;
    for (int i = 0; i < p; ++i) rot[(int64_t)jj * p + i] = sg * V[i * p + j];  // column-major: column jj
  }
}

__global__ void k_scores(const double* X, int64_t ldx, int64_t n, int p, int k, const double* mu, const double* sd,
                         int scale, const double* rot, double* scores) {
  const int64_t r = blockIdx.x * (int64_t)NT + threadIdx.x;
  const int j = blockIdx.y;
  if (r >= n || j >= k) return;
  double s = 0.0;
  for (int i = 0; i < p; ++i) {
    double z = X[(int64_t)i * ldx + r] - mu[i];
    if (scale) z = z / sd[i];
    s += z * rot[(int64_t)j * p + i];
  }
  scores[(int64_t)j * n + r] = s;
}

// ------------------------------------------------------------------ varimax (reading R25)
// One CTA: x and Z = x T resident in shared memory (column-major, ld = p).  Per
// iteration: Z = x T; c_j = sum_i Z_ij^2; B = x^T (Z^3 - Z diag(c) / p); the
// polar factor T = U V^T of B by one-sided Jacobi (warp 0: lane i holds row i
// of the working columns, cyclic sweeps until every column pair is orthogonal
// to 1e-15); d = sum of singular values; stop when d < d_past (1 + eps).
constexpr int VK = 32;  // largest k
__device__ __forceinline__ double warp_sum_d(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__global__ void k_varimax(const double* L, int64_t ldl, int p, int k, int normalize, double eps, int max_iter,
                          double* load_o, double* rot_o, int32_t* iters_o, int* bad) {
  extern __shared__ double vsm[];
  double* x = vsm;                  // p x k
  double* Z = x + (size_t)p * k;    // p x k
  double* sc = Z + (size_t)p * k;   // p
  __shared__ double T[VK * VK], B[VK * VK], A[VK * VK], Vm[VK * VK], cs[VK], sv[VK];
  __shared__ double s_d;
  __shared__ int s_stop, s_it;
  const int tid = threadIdx.x, nt = blockDim.x, lane = tid & 31, wid = tid >> 5;
  for (int e = tid; e < p * k; e += nt) x[e] = L[(int64_t)(e / p) * ldl + (e % p)];
  __syncthreads();
  if (normalize) {
    for (int i = tid; i < p; i += nt) {
      double s2 = 0.0;
      for (int j = 0; j < k; ++j) s2 += x[i + p * j] * x[i + p * j];
      sc[i] = sqrt(s2);
      if (!(sc[i] > 0.0)) atomicExch(bad, 1);
    }
    __syncthreads();
    for (int e = tid; e < p * k; e += nt) x[e] = x[e] / sc[e % p];
  }
  for (int e = tid; e < k * k; e += nt) T[e] = (e % k == e / k) ? 1.0 : 0.0;
  if (tid == 0) {
    s_d = 0.0;
    s_stop = 0;
    s_it = 0;
  }
  __syncthreads();
  for (int it = 1; it <= max_iter && k >= 2; ++it) {
    for (int e = tid; e < p * k; e += nt) {  // Z = x T
      const int i = e % p, j = e / p;
      double z = 0.0;
      for (int l = 0; l < k; ++l) z += x[i + p * l] * T[l + k * j];
      Z[e] = z;
    }
    __syncthreads();
    for (int j = wid; j < k; j += nt / 32) {  // c_j = sum_i Z_ij^2
      double c = 0.0;
      for (int i = lane; i < p; i += 32) c += Z[i + p * j] * Z[i + p * j];
      c = warp_sum_d(c);
      if (lane == 0) cs[j] = c / p;
    }
    __syncthreads();
    for (int e = tid; e < k * k; e += nt) {  // B = x^T (Z^3 - Z c / p)
      const int a = e % k, b = e / k;
      double v = 0.0;
      for (int i = 0; i < p; ++i) {
        const double z = Z[i + p * b];
        v += x[i + p * a] * (z * z * z - z * cs[b]);
      }
      B[e] = v;
      A[e] = v;
      Vm[e] = (a == b) ? 1.0 : 0.0;
    }
    __syncthreads();
    if (wid == 0) {  // one-sided Jacobi on the columns of A = B; Vm accumulates the rotations
      for (int sweep = 0; sweep < 60; ++sweep) {
        bool rotated = false;
        for (int a = 0; a < k - 1; ++a)
          for (int b = a + 1; b < k; ++b) {
            const double ua = lane < k ? A[lane + k * a] : 0.0, ub = lane < k ? A[lane + k * b] : 0.0;
            const double alpha = warp_sum_d(ua * ua), beta = warp_sum_d(ub * ub), gamma = warp_sum_d(ua * ub);
            if (fabs(gamma) > 1e-15 * sqrt(alpha * beta) && gamma != 0.0) {
              rotated = true;
              const double zeta = (beta - alpha) / (2.0 * gamma);
              const double t = (zeta >= 0.0 ? 1.0 : -1.0) / (fabs(zeta) + sqrt(1.0 + zeta * zeta));
              const double c = 1.0 / sqrt(1.0 + t * t), sn = c * t;
              if (lane < k) {
                A[lane + k * a] = c * ua - sn * ub;
                A[lane + k * b] = sn * ua + c * ub;
                const double va = Vm[lane + k * a], vb = Vm[lane + k * b];
                Vm[lane + k * a] = c * va - sn * vb;
                Vm[lane + k * b] = sn * va + c * vb;
              }
            }
            __syncwarp();
          }
        if (!rotated) break;
      }
      for (int j = 0; j < k; ++j) {  // singular values = column norms; U = A / s
        const double u = lane < k ? A[lane + k * j] : 0.0;
        const double sj = sqrt(warp_sum_d(u * u));
        if (lane == 0) sv[j] = sj;
        if (lane < k) A[lane + k * j] = sj > 0.0 ? u / sj : 0.0;
      }
      __syncwarp();
    }
    __syncthreads();
    for (int e = tid; e < k * k; e += nt) {  // T = U V^T
      const int a = e % k, b = e / k;
      double v = 0.0;
      for (int l = 0; l < k; ++l) v += A[a + k * l] * Vm[b + k * l];
      T[e] = v;
    }
    if (tid == 0) {
      double d = 0.0;
      for (int j = 0; j < k; ++j) d += sv[j];
      const double dp = s_d;
      s_d = d;
      s_it = it;
      if (d < dp * (1.0 + eps)) s_stop = 1;
    }
    __syncthreads();
    if (s_stop) break;
  }
  for (int e = tid; e < p * k; e += nt) {  // loadings = x T (rows scaled back)
    const int i = e % p, j = e / p;
    double z = 0.0;
    for (int l = 0; l < k; ++l) z += x[i + p * l] * T[l + k * j];
    load_o[e] = normalize ? z * sc[i] : z;
  }
  for (int e = tid; e < k * k; e += nt) rot_o[e] = T[e];
  if (tid == 0 && iters_o) *iters_o = s_it;
}

}  // namespace

void varimax_impl(const double* L_in, int64_t ldl, int32_t p, int32_t k, int32_t normalize, double eps,
                  double* load_o, double* rot_o, int32_t* iters_host, cudaStream_t s) {
  InStage Ls(L_in, sizeof(double) * (size_t)(ldl * (k - 1) + p), s);
  OutStage lo(load_o, sizeof(double) * (size_t)p * k, s), ro(rot_o, sizeof(double) * (size_t)k * k, s);
  DBuf<int32_t> it(1, s);
  DBuf<int> bad(1, s);
  BF_CUDA_CHECK(cudaMemsetAsync(bad.p, 0, sizeof(int), s));
  const size_t smem = sizeof(double) * (2 * (size_t)p * k + p);
  static int vmax = 0;
  if (!vmax) vmax = dyn_smem_limit(k_varimax);
  BF_REQUIRE(smem <= (size_t)vmax, BF_ENOTIMPL, "bf_varimax: p x k too large for shared memory");
  {
    KScope ks_("k_varimax", s, 0.0);
    k_varimax<<<1, 256, smem, s>>>((const double*)Ls.dptr, ldl, p, k, normalize, eps, 1000, (double*)lo.dptr,
                                   (double*)ro.dptr, it.p, bad.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  int hbad = 0;
  int32_t hit = 0;
  BF_CUDA_CHECK(cudaMemcpyAsync(&hbad, bad.p, sizeof(int), cudaMemcpyDeviceToHost, s));
  BF_CUDA_CHECK(cudaMemcpyAsync(&hit, it.p, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  lo.finish(s);
  ro.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  BF_REQUIRE(!hbad, BF_EINVAL, "bf_varimax: a row of zero loadings cannot be normalised");
  if (iters_host) *iters_host = hit;
}

// Reading R15 ("less than 10", "4 PCs ... > 97%"): the number of retained components is the
// smallest k whose cumulative share of the variance sum_j sdev_j^2 reaches frac, clamped to [1, min(cap, p)].
// One thread: p <= 1024 squares summed in index order.
__global__ void k_pca_retained(const double* __restrict__ sdev, int p, double frac, int cap, int32_t* __restrict__ k) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  double tot = 0.0;
  for (int j = 0; j < p; ++j) tot += sdev[j] * sdev[j];
  int kk = p;
  double c = 0.0;
  for (int j = 0; j < p; ++j) {
    c += sdev[j] * sdev[j];
    if (c / tot >= frac) {
      kk = j + 1;
      break;
    }
  }
  kk = kk < cap ? kk : cap;
  kk = kk < p ? kk : p;
  *k = kk < 1 ? 1 : kk;
}

void pca_retained_impl(const double* sdev_in, int32_t p, double frac, int32_t cap, int32_t* k_host, cudaStream_t s) {
  InStage sd(sdev_in, sizeof(double) * (size_t)p, s);
  DBuf<int32_t> kd(1, s);
  {
    KScope ks_("k_pca_retained", s, 0.0);
    k_pca_retained<<<1, 32, 0, s>>>((const double*)sd.dptr, p, frac, cap, kd.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  BF_CUDA_CHECK(cudaMemcpyAsync(k_host, kd.p, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

void pca_impl(const double* X_in, int64_t ldx, int64_t n, int32_t p, int32_t scale, int32_t k, double* sdev_o,
              double* rot_o, double* center_o, double* scores_o, cudaStream_t s) {
  InStage Xs(X_in, sizeof(double) * (size_t)(ldx * (p - 1) + n), s);
  const double* X = (const double*)Xs.dptr;
  OutStage sdv(sdev_o, sizeof(double) * p, s), rot(rot_o, sizeof(double) * p * p, s);
  OutStage cen(center_o, center_o ? sizeof(double) * p : 0, s);
  OutStage sco(scores_o, scores_o ? sizeof(double) * (size_t)n * k : 0, s);
  DBuf<double> mu(p, s), sd(p, s), C((size_t)p * p, s);
  {
    KScope ks_("k_colstats", s, 0.0);
    k_colstats<<<p, NT, 0, s>>>(X, ldx, n, scale, mu.p, sd.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  if (scale) {
    std::vector<double> hsd(p);
    BF_CUDA_CHECK(cudaMemcpyAsync(hsd.data(), sd.p, sizeof(double) * p, cudaMemcpyDeviceToHost, s));
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
    for (int j = 0; j < p; ++j) BF_REQUIRE(hsd[j] > 0.0, BF_EINVAL, "bf_pca: zero-variance column with scale");
  }
  const int np = p * (p + 1) / 2;
  const size_t gsm = sizeof(double) * ((size_t)GR * p + np);
  const int smax = dyn_smem_limit(k_gram);
  BF_REQUIRE(gsm <= (size_t)smax, BF_ENOTIMPL, "bf_pca: p too large for the shared-memory Gram");
  const int nparts = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, GR), 296));
  DBuf<double> part((size_t)nparts * np, s);
  {
    KScope ks_("k_gram", s, 0.0);
    k_gram<<<nparts, NT, gsm, s>>>(X, ldx, n, p, mu.p, sd.p, scale, part.p);
  }
  {
    KScope ks_("k_gram_reduce", s, 0.0);
    k_gram_reduce<<<(unsigned)ceil_div(np, NT), NT, 0, s>>>(part.p, nparts, p, n, C.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  const int P = p + (p & 1);
  const size_t jsm = sizeof(double) * (2 * (size_t)p * p + P) + sizeof(int) * P + 16;
  BF_REQUIRE(jsm <= (size_t)dyn_smem_limit(k_jacobi), BF_ENOTIMPL, "bf_pca: p too large for the shared-memory Jacobi");
  {
    KScope ks_("k_jacobi", s, 0.0);
    k_jacobi<<<1, NT, jsm, s>>>(C.p, p, (double*)sdv.dptr, (double*)rot.dptr);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  if (center_o) BF_CUDA_CHECK(cudaMemcpyAsync(cen.dptr, mu.p, sizeof(double) * p, cudaMemcpyDeviceToDevice, s));
  if (scores_o && k > 0) {
    {
      KScope ks_("k_scores", s, 0.0);
      k_scores<<<dim3((unsigned)ceil_div(n, NT), k), NT, 0, s>>>(X, ldx, n, p, k, mu.p, sd.p, scale,
                                                                 (const double*)rot.dptr, (double*)sco.dptr);
    }
    BF_CUDA_CHECK(cudaGetLastError());
  }
  sdv.finish(s);
  rot.finish(s);
  if (center_o) cen.finish(s);
  if (scores_o) sco.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

}  // namespace bf
