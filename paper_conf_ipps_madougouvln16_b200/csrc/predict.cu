// predict.cu -- batched forest prediction (P:95 step 3, S5).
//
// One thread per query row; a CTA stages its rows' predictors in shared
// memory row-major (coalesced column loads), then every thread walks all the
// forest's trees in tree order (16-byte node loads through the read-only
// path) and sums the leaf values in fp64.  All CTAs advance through the trees
// in the same order, so the trees being walked at any moment stay L2-resident.
#include <algorithm>

#include "bf_internal.cuh"

namespace bf {
namespace {

constexpr int PT = 128;   // rows per CTA
constexpr int PILP = 8;  // trees walked concurrently by one thread

__device__ __forceinline__ Node16 load_node(const Node16* p) {
  const int4 v = __ldg(reinterpret_cast<const int4*>(p));
  Node16 n;
  n.v = __hiloint2double(v.y, v.x);
  n.feature = v.z;
  n.left = v.w;
  return n;
}

// Trees [t_begin, t_end) of one tree block for every row; partial sums are
// accumulated into yhat_sum (first block writes), so leaves are still added in
// tree order.  A block of a few trees stays L2-resident while all rows walk it.
__global__ void __launch_bounds__(PT) k_predict_smem(const Node16* __restrict__ nodes, const int64_t* __restrict__ off,
                                                     int32_t t_begin, int32_t t_end, int first, int last,
                                                     const double* __restrict__ Xq, int64_t ldq,
                                                     int64_t m, int p, double* yhat_sum, double* yhat, double inv_t,
                                                     unsigned long long* visits) {
  extern __shared__ double sx[];  // PT x p, row-major, padded stride p|1
  const int stride = p | 1;
  const int64_t r0 = (int64_t)blockIdx.x * PT;
  const int rows = (int)(m - r0 < PT ? m - r0 : PT);
  {  // stage the tile: every thread's column loads in flight together (16 at a time)
    const int r = threadIdx.x;
    const bool ok = r < rows;
    const double* src = Xq + r0 + (ok ? r : 0);
    for (int f0 = 0; f0 < p; f0 += 16) {
      double v[16];
#pragma unroll
      for (int u = 0; u < 16; ++u) v[u] = (f0 + u < p) ? __ldcs(src + (int64_t)(f0 + u) * ldq) : 0.0;
#pragma unroll
      for (int u = 0; u < 16; ++u)
        if (f0 + u < p && ok) sx[r * stride + f0 + u] = v[u];
    }
  }
  __syncthreads();
  if ((int)threadIdx.x >= rows) return;
  const double* x = sx + threadIdx.x * stride;
  const int64_t rr = r0 + threadIdx.x;
  double acc = first ? 0.0 : yhat_sum[rr];
  unsigned long long nv = 0;
  // ILP trees walked together (independent dependency chains; the last group
  // of a block is masked); leaf values are added in tree order, as in S5
  for (int32_t t = t_begin; t < t_end; t += PILP) {
    const int na = t_end - t < PILP ? t_end - t : PILP;
    const Node16* tn[PILP];
    Node16 nd[PILP];
#pragma unroll
    for (int u = 0; u < PILP; ++u) {
      tn[u] = nodes + off[t + (u < na ? u : 0)];
      nd[u] = load_node(tn[u]);
      if (u >= na) nd[u].feature = -1;
    }
    nv += na;
    bool any = true;
    while (any) {
      any = false;
#pragma unroll
      for (int u = 0; u < PILP; ++u)
        if (nd[u].feature >= 0) {
          nd[u] = load_node(tn[u] + (x[nd[u].feature] <= nd[u].v ? nd[u].left : nd[u].left + 1));
          ++nv;
          any = true;
        }
    }
#pragma unroll
    for (int u = 0; u < PILP; ++u)
      if (u < na) acc += nd[u].v;
  }
  if (visits) atomicAdd(visits, nv);
  yhat_sum[rr] = acc;
  if (last && yhat) yhat[rr] = acc * inv_t;
}

__global__ void __launch_bounds__(PT) k_predict_gmem(const Node16* __restrict__ nodes, const int64_t* __restrict__ off,
                                                     int32_t ntrees, const double* __restrict__ Xq, int64_t ldq,
                                                     int64_t m, double* yhat_sum, double* yhat, double inv_t,
                                                     unsigned long long* visits) {
  const int64_t r = (int64_t)blockIdx.x * PT + threadIdx.x;
  if (r >= m) return;
  double acc = 0.0;
  unsigned long long nv = 0;
  for (int32_t t = 0; t < ntrees; ++t) {
    const Node16* tn = nodes + off[t];
    Node16 nd = load_node(tn);
    ++nv;
    while (nd.feature >= 0) {
      nd = load_node(tn + (__ldg(Xq + (int64_t)nd.feature * ldq + r) <= nd.v ? nd.left : nd.left + 1));
      ++nv;
    }
    acc += nd.v;
  }
  if (visits) atomicAdd(visits, nv);
  if (yhat_sum) yhat_sum[r] = acc;
  if (yhat) yhat[r] = acc * inv_t;
}

}  // namespace

void predict_impl(const bf_forest* f, const double* Xq_in, int64_t ldq, int64_t m, double* ys_in, double* yh_in,
                  int32_t ntree_total, cudaStream_t s) {
  if (m == 0) return;
  const int p = f->info.p;
  const int32_t nt = f->info.tree_end - f->info.tree_begin;
  InStage Xs(Xq_in, sizeof(double) * (size_t)(ldq * (p - 1) + m), s);
  OutStage ys(ys_in, ys_in ? sizeof(double) * m : 0, s), yh(yh_in, yh_in ? sizeof(double) * m : 0, s);
  const double inv_t = 1.0 / (double)(ntree_total > 0 ? ntree_total : std::max(nt, 1));
  const unsigned grid = (unsigned)ceil_div(m, PT);
  const size_t smem = sizeof(double) * (size_t)PT * (size_t)(p | 1);
  static int smax = 0;
  if (!smax) smax = dyn_smem_limit(k_predict_smem);
  DBuf<unsigned long long> vis;
  if (prof_enabled()) {
    vis.alloc(1, s);
    BF_CUDA_CHECK(cudaMemsetAsync(vis.p, 0, 8, s));
  }
  if (smem <= (size_t)smax) {
    // tree blocks of <= 64 MB of nodes (L2-resident while every row walks them)
    double* ysum = ys_in ? (double*)ys.dptr : nullptr;
    DBuf<double> ytmp;
    if (!ysum) {
      ytmp.alloc(m, s);
      ysum = ytmp.p;
    }
    const int64_t block_bytes = 64ll << 20;
    int32_t t0 = 0;
    while (t0 < nt || (nt == 0 && t0 == 0)) {
      int32_t t1 = t0 + 1;
      while (t1 < nt && (f->tree_off[t1 + 1] - f->tree_off[t0]) * (int64_t)sizeof(Node16) <= block_bytes) ++t1;
      if (t1 < nt && t1 - t0 > PILP) t1 = t0 + (t1 - t0) / PILP * PILP;  // whole ILP groups
      if (nt == 0) t1 = 0;
      {
        KScope ks_("k_predict_smem", s, 0.0);
        k_predict_smem<<<grid, PT, smem, s>>>(f->d_nodes, f->d_tree_off, t0, t1, t0 == 0, t1 >= nt,
                                             (const double*)Xs.dptr, ldq, m, p, ysum,
                                             yh_in ? (double*)yh.dptr : nullptr, inv_t, vis.p);
      }
      if (nt == 0) break;
      t0 = t1;
    }
  } else {
    {
      KScope ks_("k_predict_gmem", s, 0.0);
      k_predict_gmem<<<grid, PT, 0, s>>>(f->d_nodes, f->d_tree_off, nt, (const double*)Xs.dptr, ldq, m,
                                       ys_in ? (double*)ys.dptr : nullptr, yh_in ? (double*)yh.dptr : nullptr, inv_t, vis.p);
    }
  }
  BF_CUDA_CHECK(cudaGetLastError());
  if (vis.p) {  // profile mode: algorithmic bytes = node visits x 16 B + rows x (8p + 16) B
    unsigned long long hv = 0;
    BF_CUDA_CHECK(cudaMemcpyAsync(&hv, vis.p, 8, cudaMemcpyDeviceToHost, s));
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
    prof_add_bytes(smem <= (size_t)smax ? "k_predict_smem" : "k_predict_gmem",
                   16.0 * (double)hv + (double)m * (8.0 * p + 16.0 * ((ys_in != nullptr) + (yh_in != nullptr))));
  }
  if (ys_in) ys.finish(s);
  if (yh_in) yh.finish(s);
  if (ys.host || yh.host || Xs.tmp.p) BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

}  // namespace bf
