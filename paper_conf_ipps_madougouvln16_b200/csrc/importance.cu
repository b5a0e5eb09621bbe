// importance.cu -- OOB prediction and permutation importance (SURVEY 8(a)
// rows a13-a15; S6-S8).
//
// Per batch of trees: regenerate the bootstrap (Philox BOOT, identical to
// the fit), compact each tree's OOB rows in ascending order, then one thread
// per (tree, OOB row a):
//   * walk the tree -> f_t(x_a); accumulate e_t, oob_sum, oob_cnt;
//   * for every predictor m tested on that path (first occurrence only) walk
//     again from that node with x_m replaced by x_{O_t[pi_tm(a)], m}.  A path
//     that does not test m gives the same leaf, so its contribution to
//     e_tm - e_t is exactly zero and is skipped; predictors never used by the
//     tree get d_tm = 0 exactly (S7).
#include <algorithm>
#include <cstdlib>

#include "bf_internal.cuh"

namespace bf {
namespace {

constexpr int NT = 256;
constexpr int OCH = 4096;  // rows per CTA chunk in the OOB compaction

__device__ __forceinline__ Node16 ld_node(const Node16* p) {
  const int4 v = __ldg(reinterpret_cast<const int4*>(p));
  Node16 n;
  n.v = __hiloint2double(v.y, v.x);
  n.feature = v.z;
  n.left = v.w;
  return n;
}

// S7 Feistel permutation pi_tm on [0, n_o) with cycle walking.
__device__ __forceinline__ int64_t feistel(uint64_t seed, uint32_t t, uint32_t m, int64_t n_o, int64_t a) {
  int b = 64 - __clzll((unsigned long long)(n_o - 1));  // ceil(log2 n_o) for n_o >= 2; 0 for n_o == 1
  if (n_o <= 1) b = 0;
  if (b < 2) b = 2;
  b += b & 1;
  const int h = b >> 1;
  const uint32_t mask = (uint32_t)((1ull << h) - 1ull);
  uint64_t v = (uint64_t)a;
  do {
    uint32_t L = (uint32_t)(v >> h), R = (uint32_t)(v & mask);
#pragma unroll 1
    for (uint32_t r = 0; r < 6; ++r) {
      uint32_t x[4];
      philox4x32_10(R, r, 3u | (m << 8), t, (uint32_t)seed, (uint32_t)(seed >> 32), x);
      const uint32_t nR = L ^ (x[0] & mask);
      L = R;
      R = nR;
    }
    v = ((uint64_t)L << h) | R;
  } while ((int64_t)v >= n_o);
  return (int64_t)v;
}

// pi_tm for every OOB position of a batch, precomputed per (tree, predictor):
// perm[(b * p + m) * n + a] = pi_tm(a), a < n_o.  The Feistel round function
// F_r(R) only takes h-bit inputs (h = b/2), so for h <= 12 a CTA first fills
// the 6 x 2^h round values of its (t, m) in shared memory (6 x 2^h Philox
// calls) and every pi(a) is then 6 shared-memory lookups per cycle-walking
// step; otherwise F is computed on the fly.  Same values as feistel().
constexpr int PH_MAX = 12;
__device__ __forceinline__ int feistel_h(int64_t n_o) {
  int b = 64 - __clzll((unsigned long long)(n_o - 1));
  if (n_o <= 1) b = 0;
  if (b < 2) b = 2;
  b += b & 1;
  return b >> 1;
}
// Round tables of the batch, computed once per (tree, predictor): gtab[(b * p + m) * tstride + r * 2^h + R] =
// F_r(R) & mask (h = feistel_h(n_o) <= PH_MAX); every k_perm_fill CTA of (b, m) copies its table from L2.
__global__ void k_ftab_fill(uint64_t seed, int32_t t0, int p, const int64_t* nout, int tstride, uint32_t* gtab) {
  const int b = blockIdx.z, m = blockIdx.y;
  const int64_t n_o = nout[b];
  if (n_o <= 0) return;
  const int h = feistel_h(n_o);
  if (h > PH_MAX) return;
  const int S = 1 << h;
  const uint32_t mask = (uint32_t)S - 1u, t = (uint32_t)(t0 + b);
  uint32_t* out = gtab + ((int64_t)b * p + m) * tstride;
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < 6 * S; k += gridDim.x * blockDim.x) {
    uint32_t x[4];
    philox4x32_10((uint32_t)(k & (S - 1)), (uint32_t)(k >> h), 3u | ((uint32_t)m << 8), t, (uint32_t)seed,
                  (uint32_t)(seed >> 32), x);
    out[k] = x[0] & mask;
  }
}

__global__ void __launch_bounds__(512) k_perm_fill(uint64_t seed, int32_t t0, int p, int64_t n, const int64_t* nout,
                                                   const uint32_t* gtab, int tstride, int32_t* perm,
                                                   const uint8_t* used) {
  extern __shared__ uint32_t ftab[];  // 6 x 2^h (h <= PH_MAX)
  const int b = blockIdx.z, m = blockIdx.y;
  const int64_t n_o = nout[b];
  if (n_o <= 0) return;
  // a predictor no split of the tree uses is never re-walked (S7: its d_tm is 0): no permutation needed
  if (!used[(int64_t)b * p + m]) return;
  const uint32_t t = (uint32_t)(t0 + b);
  const int h = feistel_h(n_o);
  const uint32_t mask = (uint32_t)((1ull << h) - 1ull);
  const bool tab = h <= PH_MAX;
  if (tab) {  // F_r(R) & mask for every round r and h-bit input R (k_ftab_fill)
    const uint32_t* src = gtab + ((int64_t)b * p + m) * tstride;
    for (int k = threadIdx.x; k < (6 << h); k += blockDim.x) ftab[k] = src[k];
    __syncthreads();
  }
  int32_t* out = perm + ((int64_t)b * p + m) * n;
  const int64_t step = (int64_t)gridDim.x * blockDim.x;
  if (!tab) {
    for (int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; a < n_o; a += step)
      out[a] = (int32_t)feistel(seed, t, (uint32_t)m, n_o, a);
    return;
  }
  // 2h <= 2 * PH_MAX bits: 32-bit arithmetic throughout (n_o < 2^31).  Cycle walking needs ~2.9 Feistel
  // passes per value on average (the domain 2^2h is up to ~3x n_o) but the slowest lane of a warp needs ~9:
  // each lane therefore walks its own sequence of positions one pass at a time and moves on to its next
  // position as soon as the current one lands in [0, n_o), so no lane waits for the warp's slowest walk.
  const uint32_t* f0 = ftab;
  const uint32_t* f1 = f0 + (1u << h);
  const uint32_t* f2 = f1 + (1u << h);
  const uint32_t* f3 = f2 + (1u << h);
  const uint32_t* f4 = f3 + (1u << h);
  const uint32_t* f5 = f4 + (1u << h);
  const uint32_t no = (uint32_t)n_o;
  int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  uint32_t v = (uint32_t)a;
  while (a < n_o) {
    uint32_t L = v >> h, R = v & mask;
    L ^= f0[R];
    R ^= f1[L];
    L ^= f2[R];
    R ^= f3[L];
    L ^= f4[R];
    R ^= f5[L];
    v = (L << h) | R;  // six rounds (L, R) <- (R, L ^ F_r(R)) end with the halves back in place
    if (v < no) {
      out[a] = (int32_t)v;
      a += step;
      v = (uint32_t)a;
    }
  }
}

__global__ void k_perm(uint64_t seed, int32_t t, int32_t m, int64_t n_o, int64_t* out) {
  const int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (a < n_o) out[a] = feistel(seed, (uint32_t)t, (uint32_t)m, n_o, a);
}

__global__ void k_oob_count(const int32_t* w, int64_t n, int nchunk, int32_t* cnt) {
  __shared__ int32_t sm[NT / 32];
  const int c = blockIdx.x, b = blockIdx.y;
  int32_t k = 0;
  for (int u = threadIdx.x; u < OCH; u += NT) {
    const int64_t i = (int64_t)c * OCH + u;
    if (i < n) k += w[(int64_t)b * n + i] == 0;
  }
  for (int o = 16; o > 0; o >>= 1) k += __shfl_down_sync(0xffffffffu, k, o);
  if ((threadIdx.x & 31) == 0) sm[threadIdx.x >> 5] = k;
  __syncthreads();
  if (threadIdx.x == 0) {
    int32_t s = 0;
    for (int j = 0; j < NT / 32; ++j) s += sm[j];
    cnt[(int64_t)b * nchunk + c] = s;
  }
}

__global__ void k_oob_prefix(int32_t* cnt, int B, int nchunk, int64_t* nout) {
  const int b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= B) return;
  int32_t acc = 0;
  for (int c = 0; c < nchunk; ++c) {
    const int32_t v = cnt[(int64_t)b * nchunk + c];
    cnt[(int64_t)b * nchunk + c] = acc;
    acc += v;
  }
  nout[b] = acc;
}

__global__ void k_oob_scatter(const int32_t* w, int64_t n, int nchunk, const int32_t* cnt, uint32_t* O) {
  __shared__ int32_t sm[NT / 32];
  const int c = blockIdx.x, b = blockIdx.y;
  constexpr int V = OCH / NT;
  const int64_t i0 = (int64_t)c * OCH + (int64_t)threadIdx.x * V;
  bool keep[V];
  int32_t k = 0;
#pragma unroll
  for (int u = 0; u < V; ++u) {
    keep[u] = (i0 + u < n) && w[(int64_t)b * n + i0 + u] == 0;
    k += keep[u];
  }
  // block exclusive scan
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int32_t inc = k;
  for (int o = 1; o < 32; o <<= 1) {
    const int32_t v = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += v;
  }
  if (lane == 31) sm[wid] = inc;
  __syncthreads();
  if (threadIdx.x == 0)
    for (int j = 1; j < NT / 32; ++j) sm[j] += sm[j - 1];
  __syncthreads();
  int32_t pre = inc - k + (wid ? sm[wid - 1] : 0) + cnt[(int64_t)b * nchunk + c];
  uint32_t* Ob = O + (int64_t)b * n;
#pragma unroll
  for (int u = 0; u < V; ++u)
    if (keep[u]) Ob[pre++] = (uint32_t)(i0 + u);
}

// IncNodePurity slots: sum of drss of splits on m, per local tree.
// (per-CTA shared-memory histogram over the predictors, one global atomic per (CTA, predictor))
// IncNodePurity slots of the batch's trees and the predictors each tree splits on (used[b * p + m] = 1;
// zero-initialised by the caller).
__global__ void k_npur(const Node16* nodes, const double* drss, const int64_t* off, int32_t i0, int p, double* npur,
                       uint8_t* used) {
  extern __shared__ double hp[];  // p doubles, then p flags
  int* hu = reinterpret_cast<int*>(hp + p);
  const int b = blockIdx.y;
  const int32_t i = i0 + b;
  for (int f = threadIdx.x; f < p; f += NT) {
    hp[f] = 0.0;
    hu[f] = 0;
  }
  __syncthreads();
  const int64_t lo = off[i], hi = off[i + 1];
  for (int64_t k = lo + blockIdx.x * (int64_t)NT + threadIdx.x; k < hi; k += (int64_t)gridDim.x * NT) {
    const int f = nodes[k].feature;
    if (f >= 0) {
      atomicAdd(&hp[f], drss[k]);
      atomicExch(&hu[f], 1);
    }
  }
  __syncthreads();
  for (int f = threadIdx.x; f < p; f += NT) {
    if (hp[f] != 0.0) atomicAdd(&npur[(int64_t)i * p + f], hp[f]);
    if (hu[f]) used[(int64_t)b * p + f] = 1;
  }
}

struct ImpArgs {
  const Node16* nodes;
  const int64_t* off;
  const double* X;
  int64_t ldx;
  const double* y;
  int64_t n;
  int p;
  uint64_t seed;
  int32_t tree_begin;  // global id of local tree 0
  int32_t i0;          // local index of batch tree 0
  const uint32_t* O;   // batch OOB lists, stride n
  const int64_t* nout; // batch OOB counts
  double* d_slots;     // local tree slots
  double* oob_sum;
  int32_t* oob_cnt;
  double* e_t;
  const int32_t* perm;  // pi_tm(a) of the batch (k_perm_fill), stride n per (tree, predictor)
};

constexpr int IPT = 128;  // OOB rows per CTA (one thread each; their predictors staged in shared memory)
constexpr int IPT_WIDE = 32;  // rows per CTA of the Node16 kernel when p is too large for a 128-row tile
constexpr int ILP = 4;    // permuted walks interleaved per thread

// One CTA = IPT consecutive OOB positions a of one tree.  The rows' predictors
// are staged row-major in shared memory (coalesced column loads of the
// ascending OOB rows), so every walk reads x from shared memory and only the
// node array (L2-resident: the CTAs of one tree run together) and the
// permuted value x_{O_t[pi(a)], m} come from global memory.  The first
// occurrences of each predictor on the original path are collected ILP at a
// time and their re-walks run interleaved (independent dependency chains).
template <int TP>  // OOB rows per CTA: TP, or TP_WIDE when a 128-row fp64 tile exceeds shared memory (large p)
__global__ void __launch_bounds__(TP) k_importance(ImpArgs g) {
  extern __shared__ double ism[];  // sacc[p] | x tile TP x (p|1)
  double* sacc = ism;
  const int stride = g.p | 1;
  double* sx = ism + ((g.p + 1) & ~1);
  __shared__ double serr[TP / 32];
  const int b = blockIdx.y;
  const int32_t i = g.i0 + b;
  const uint32_t t = (uint32_t)(g.tree_begin + i);
  const int64_t n_o = g.nout[b];
  const int64_t a0 = (int64_t)blockIdx.x * TP;
  if (a0 >= n_o) return;  // uniform per CTA
  for (int m = threadIdx.x; m < g.p; m += TP) sacc[m] = 0.0;
  const uint32_t* Ob = g.O + (int64_t)b * g.n;
  const int64_t a = a0 + threadIdx.x;
  const bool act = a < n_o;
  const uint32_t r = act ? Ob[a] : Ob[a0];
  {  // stage the tile: 16 column loads in flight per thread
    double* xs = sx + threadIdx.x * stride;
    for (int f0 = 0; f0 < g.p; f0 += 16) {
      double v[16];
#pragma unroll
      for (int u = 0; u < 16; ++u) v[u] = (f0 + u < g.p) ? __ldg(g.X + (int64_t)(f0 + u) * g.ldx + r) : 0.0;
#pragma unroll
      for (int u = 0; u < 16; ++u)
        if (f0 + u < g.p) xs[f0 + u] = v[u];
    }
  }
  __syncthreads();
  double err0 = 0.0;
  if (act) {
    const double* x = sx + threadIdx.x * stride;
    const Node16* tn = g.nodes + g.off[i];
    const double yr = g.y[r];
    // original walk
    Node16 nd = ld_node(tn);
    while (nd.feature >= 0) nd = ld_node(tn + (x[nd.feature] <= nd.v ? nd.left : nd.left + 1));
    const double f0 = nd.v;
    const double d0 = yr - f0;
    err0 = d0 * d0;
    atomicAdd(&g.oob_sum[r], f0);
    atomicAdd(&g.oob_cnt[r], 1);
    // permuted walks from the first occurrence of each predictor on the path
    uint64_t seen = 0;
    int depth = 0;
    nd = ld_node(tn);
    for (;;) {
      int cnt = 0;
      int qm[ILP];
      Node16 q[ILP];
      while (nd.feature >= 0 && cnt < ILP) {
        const int m = nd.feature;
        bool first = !((seen >> (m & 63)) & 1ull);
        if (!first && g.p > 64) {  // bitmask collision possible: verify on the path prefix
          first = true;
          int kk = 0;
          for (int d = 0; d < depth; ++d) {
            const Node16 pq = ld_node(tn + kk);
            if (pq.feature == m) {
              first = false;
              break;
            }
            kk = x[pq.feature] <= pq.v ? pq.left : pq.left + 1;
          }
        }
        seen |= 1ull << (m & 63);
        if (first) {
#pragma unroll
          for (int u = 0; u < ILP; ++u)
            if (u == cnt) {
              qm[u] = m;
              q[u] = nd;
            }
          ++cnt;
        }
        nd = ld_node(tn + (x[m] <= nd.v ? nd.left : nd.left + 1));
        ++depth;
      }
      if (cnt == 0) break;
      double xm[ILP];
#pragma unroll
      for (int u = 0; u < ILP; ++u) {
        if (u < cnt) {
          const int64_t pa = __ldg(g.perm + ((int64_t)b * g.p + qm[u]) * g.n + a);
          xm[u] = __ldg(g.X + (int64_t)qm[u] * g.ldx + Ob[pa]);
        } else {
          q[u].feature = -1;
          qm[u] = -1;
          xm[u] = 0.0;
        }
      }
      bool any = true;
      while (any) {
        any = false;
#pragma unroll
        for (int u = 0; u < ILP; ++u)
          if (q[u].feature >= 0) {
            const double xv = q[u].feature == qm[u] ? xm[u] : x[q[u].feature];
            q[u] = ld_node(tn + (xv <= q[u].v ? q[u].left : q[u].left + 1));
            any = true;
          }
      }
#pragma unroll
      for (int u = 0; u < ILP; ++u)
        if (u < cnt) {
          const double d1 = yr - q[u].v;
          const double diff = d1 * d1 - err0;
          if (diff != 0.0) atomicAdd(&sacc[qm[u]], diff);
        }
    }
  }
  // e_t
  for (int o = 16; o > 0; o >>= 1) err0 += __shfl_down_sync(0xffffffffu, err0, o);
  if ((threadIdx.x & 31) == 0) serr[threadIdx.x >> 5] = err0;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int j = 0; j < TP / 32; ++j) s += serr[j];
    if (s != 0.0) atomicAdd(&g.e_t[i], s);
  }
  for (int m = threadIdx.x; m < g.p; m += TP)
    if (sacc[m] != 0.0) atomicAdd(&g.d_slots[(int64_t)i * g.p + m], sacc[m]);
}

// Row-major RN_f32 copy of the column-major X (stride xfs floats, a multiple of 4): 32 x 32 tiles through shared
// memory, coalesced on both sides.
__global__ void k_xf_rows(const double* __restrict__ X, int64_t ldx, int64_t n, int p, float* __restrict__ Xf, int xfs) {
  __shared__ float t[32][33];
  const int64_t r0 = (int64_t)blockIdx.x * 32;
  const int f0 = blockIdx.y * 32;
  for (int j = threadIdx.y; j < 32; j += blockDim.y) {  // j: feature in the tile, threadIdx.x: row
    const int64_t r = r0 + threadIdx.x;
    const int f = f0 + j;
    t[j][threadIdx.x] = (r < n && f < p) ? __double2float_rn(X[(int64_t)f * ldx + r]) : 0.0f;
  }
  __syncthreads();
  for (int j = threadIdx.y; j < 32; j += blockDim.y) {  // j: row in the tile, threadIdx.x: feature
    const int64_t r = r0 + j;
    const int f = f0 + threadIdx.x;
    if (r < n && f < xfs) Xf[r * xfs + f] = f < p ? t[threadIdx.x][j] : 0.0f;
  }
}

// k_importance8: k_importance on the compact nodes (predict.cu k_pack8) with a float row tile: the same
// walks, exact by the float-tie fallback of S5 (the fp64 x of the row from X, or the fp64 permuted value,
// against the fp64 threshold of Node16).  Half the shared memory per row (twice the CTAs per SM) and half
// the node bytes.
struct Imp8Args {
  ImpArgs a;
  const float* Xf;  // row-major RN_f32 copy of X, stride xfs (k_xf_rows): a row's tile is 4 p contiguous bytes
  int xfs;
  const uint2* nodes8;
  const uint32_t* roots8;  // per local tree (forest numbering)
  unsigned long long* prof;  // profile mode: [0] node loads, [1] permuted re-walks (algorithmic bytes), else NULL
};

__global__ void __launch_bounds__(IPT) k_importance8(Imp8Args g8) {
  const ImpArgs& g = g8.a;
  extern __shared__ double ism[];  // sacc[p] | float x tile IPT x (p|1)
  double* sacc = ism;
  const int stride = g.p | 1;
  float* sx = reinterpret_cast<float*>(ism + ((g.p + 1) & ~1));
  __shared__ double serr[IPT / 32];
  const int b = blockIdx.y;
  const int32_t i = g.i0 + b;
  const int64_t n_o = g.nout[b];
  const int64_t a0 = (int64_t)blockIdx.x * IPT;
  if (a0 >= n_o) return;  // uniform per CTA
  for (int m = threadIdx.x; m < g.p; m += IPT) sacc[m] = 0.0;
  const uint32_t* Ob = g.O + (int64_t)b * g.n;
  const int64_t a = a0 + threadIdx.x;
  const bool act = a < n_o;
  const uint32_t r = act ? Ob[a] : Ob[a0];
  {  // stage the tile from the row-major float copy: the row's 4 p bytes as 16-byte loads, 8 in flight
    float* xs = sx + threadIdx.x * stride;
    const float4* src = reinterpret_cast<const float4*>(g8.Xf + (int64_t)r * g8.xfs);
    const int nq = (g.p + 3) >> 2;
    for (int q0 = 0; q0 < nq; q0 += 8) {
      float4 v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) v[u] = (q0 + u < nq) ? __ldg(src + q0 + u) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int f = 4 * (q0 + u);
        if (f < g.p) xs[f] = v[u].x;
        if (f + 1 < g.p) xs[f + 1] = v[u].y;
        if (f + 2 < g.p) xs[f + 2] = v[u].z;
        if (f + 3 < g.p) xs[f + 3] = v[u].w;
      }
    }
  }
  __syncthreads();
  double err0 = 0.0;
  if (act) {
    const float* xs = sx + threadIdx.x * stride;
    const double* xg = g.X + r;
    const uint2* n8 = g8.nodes8;
    const Node16* n16 = g.nodes;
    const uint32_t rw = __ldg(g8.roots8 + i);
    const uint32_t root = rw & ~ROOT_LEAF;
    const double yr = g.y[r];
    uint32_t nld = 1, nrw = 0;  // node loads, re-walks (profile counters)
    // child of internal node (gid, w) for this row, feature pm (if tested) taking the value (xpf, xpd)
    auto child = [&](uint32_t gid, uint2 w, int pm, float xpf, double xpd, bool& leaf) -> uint32_t {
      const uint32_t f = n8_feature(w);
      const bool pf = (int)f == pm;
      const float xf = pf ? xpf : xs[f], tf = __uint_as_float(w.x);
      uint32_t right = xf > tf;
      if (xf == tf || xf != xf) {  // float tie: decide in fp64 (S5)
        const double xd = pf ? xpd : __ldg(xg + (int64_t)f * g.ldx);
        right = !(xd <= __ldg(&n16[gid].v));
      }
      leaf = (w.y >> (31 - right)) & 1u;
      return gid + n8_rel(w) + right;
    };
    // original walk
    double f0v;
    if (rw & ROOT_LEAF) {
      f0v = leaf8(__ldg(n8 + root));
    } else {
      uint32_t gid = root;
      uint2 w = __ldg(n8 + gid);
      for (;;) {
        bool leaf;
        const uint32_t c = child(gid, w, -1, 0.f, 0.0, leaf);
        const uint2 ch = __ldg(n8 + c);
        ++nld;
        if (leaf) {
          f0v = leaf8(ch);
          break;
        }
        gid = c;
        w = ch;
      }
    }
    const double d0 = yr - f0v;
    err0 = d0 * d0;
    atomicAdd(&g.oob_sum[r], f0v);
    atomicAdd(&g.oob_cnt[r], 1);
    // permuted walks from the first occurrence of each predictor on the path
    if (!(rw & ROOT_LEAF)) {
      uint64_t seen = 0;
      int depth = 0;
      uint32_t gid = root;
      uint2 w = __ldg(n8 + gid);
      bool at_leaf = false;
      for (;;) {
        int cnt = 0;
        int qm[ILP];
        uint32_t qg[ILP];
        uint2 qw[ILP];
        while (!at_leaf && cnt < ILP) {
          const int m = (int)n8_feature(w);
          bool first = !((seen >> (m & 63)) & 1ull);
          if (!first && g.p > 64) {  // bitmask collision possible: verify on the path prefix
            first = true;
            uint32_t kg = root;
            for (int d = 0; d < depth; ++d) {
              const uint2 pw = __ldg(n8 + kg);
              if ((int)n8_feature(pw) == m) {
                first = false;
                break;
              }
              bool lf;
              kg = child(kg, pw, -1, 0.f, 0.0, lf);
            }
          }
          seen |= 1ull << (m & 63);
          if (first) {
#pragma unroll
            for (int u = 0; u < ILP; ++u)
              if (u == cnt) {
                qm[u] = m;
                qg[u] = gid;
                qw[u] = w;
              }
            ++cnt;
          }
          bool leaf;
          const uint32_t c = child(gid, w, -1, 0.f, 0.0, leaf);
          if (leaf) {
            at_leaf = true;
          } else {
            gid = c;
            w = __ldg(n8 + c);
            ++nld;
          }
          ++depth;
        }
        if (cnt == 0) break;
        nrw += cnt;
        double xm[ILP];
        float xmf[ILP];
        bool live[ILP];
#pragma unroll
        for (int u = 0; u < ILP; ++u) {
          live[u] = u < cnt;
          xm[u] = 0.0;
          if (live[u]) {
            const int64_t pa = __ldg(g.perm + ((int64_t)b * g.p + qm[u]) * g.n + a);
            xm[u] = __ldg(g.X + (int64_t)qm[u] * g.ldx + Ob[pa]);
          } else {
            qm[u] = -1;
          }
          xmf[u] = __double2float_rn(xm[u]);
        }
        double val[ILP];
        bool any = true;
        while (any) {
          any = false;
#pragma unroll
          for (int u = 0; u < ILP; ++u)
            if (live[u]) {
              bool leaf;
              const uint32_t c = child(qg[u], qw[u], qm[u], xmf[u], xm[u], leaf);
              const uint2 ch = __ldg(n8 + c);
              ++nld;
              if (leaf) {
                val[u] = leaf8(ch);
                live[u] = false;
              } else {
                qg[u] = c;
                qw[u] = ch;
                any = true;
              }
            }
        }
#pragma unroll
        for (int u = 0; u < ILP; ++u)
          if (u < cnt) {
            const double d1 = yr - val[u];
            const double diff = d1 * d1 - err0;
            if (diff != 0.0) atomicAdd(&sacc[qm[u]], diff);
          }
      }
    }
    if (g8.prof) {  // one atomic pair per warp
      const unsigned act_m = __activemask();
      const uint32_t wl = __reduce_add_sync(act_m, nld), wr = __reduce_add_sync(act_m, nrw);
      if ((threadIdx.x & 31) == __ffs(act_m) - 1) {
        atomicAdd(&g8.prof[0], (unsigned long long)wl);
        atomicAdd(&g8.prof[1], (unsigned long long)wr);
      }
    }
  }
  // e_t
  for (int o = 16; o > 0; o >>= 1) err0 += __shfl_down_sync(0xffffffffu, err0, o);
  if ((threadIdx.x & 31) == 0) serr[threadIdx.x >> 5] = err0;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int j = 0; j < IPT / 32; ++j) s += serr[j];
    if (s != 0.0) atomicAdd(&g.e_t[i], s);
  }
  for (int m = threadIdx.x; m < g.p; m += IPT)
    if (sacc[m] != 0.0) atomicAdd(&g.d_slots[(int64_t)i * g.p + m], sacc[m]);
}


// k_importance32: k_importance8's walks on the two-level 32-byte groups (predict.cu g32_get): one 256-bit load
// decides two levels.  A permuted re-walk starts at the first node of the path that tests its predictor m: a
// group's node k (even depth), or the group's chosen child c (odd depth; then k does not test m, so the walk
// keeps the original decision at k).  Decisions are exactly S5's (float, then fp64 on a float tie: the row's
// fp64 x from X, or the fp64 permuted value, against Node16's threshold by id).  p <= 64 (one bit per predictor
// in the first-occurrence mask; wider forests take k_importance8).
struct Imp32Args {
  ImpArgs a;
  const float* Xf;
  int xfs;
  const ulonglong4* g32;
  const uint32_t* roots32;   // per local tree: root slot | ROOT_LEAF
  unsigned long long* prof;  // profile mode: [0] group loads, [1] permuted re-walks, else NULL
};

template <int IL>
__global__ void __launch_bounds__(IPT) k_importance32(Imp32Args g3) {
  const ImpArgs& g = g3.a;
  extern __shared__ double ism[];  // sacc[p] | float x tile IPT x (p|1)
  double* sacc = ism;
  const int stride = g.p | 1;
  float* sx = reinterpret_cast<float*>(ism + ((g.p + 1) & ~1));
  __shared__ double serr[IPT / 32];
  const int b = blockIdx.y;
  const int32_t i = g.i0 + b;
  const int64_t n_o = g.nout[b];
  const int64_t a0 = (int64_t)blockIdx.x * IPT;
  if (a0 >= n_o) return;  // uniform per CTA
  for (int m = threadIdx.x; m < g.p; m += IPT) sacc[m] = 0.0;
  const uint32_t* Ob = g.O + (int64_t)b * g.n;
  const int64_t a = a0 + threadIdx.x;
  const bool act = a < n_o;
  const uint32_t r = act ? Ob[a] : Ob[a0];
  {  // stage the tile from the row-major float copy: the row's 4 p bytes as 16-byte loads, 8 in flight
    float* xs = sx + threadIdx.x * stride;
    const float4* src = reinterpret_cast<const float4*>(g3.Xf + (int64_t)r * g3.xfs);
    const int nq = (g.p + 3) >> 2;
    for (int q0 = 0; q0 < nq; q0 += 8) {
      float4 v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) v[u] = (q0 + u < nq) ? __ldg(src + q0 + u) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int f = 4 * (q0 + u);
        if (f < g.p) xs[f] = v[u].x;
        if (f + 1 < g.p) xs[f + 1] = v[u].y;
        if (f + 2 < g.p) xs[f + 2] = v[u].z;
        if (f + 3 < g.p) xs[f + 3] = v[u].w;
      }
    }
  }
  __syncthreads();
  double err0 = 0.0;
  if (act) {
    const float* xs = sx + threadIdx.x * stride;
    const double* xg = g.X + r;
    const ulonglong4* G32 = g3.g32;
    const Node16* n16 = g.nodes;
    const uint32_t rw = __ldg(g3.roots32 + i);
    const uint32_t root = rw & ~ROOT_LEAF;
    const double yr = g.y[r];
    uint32_t nld = 1, nrw = 0;
    // S5 decision (1 = right) at a node of feature f, float threshold tf, Node16 id; predictor pm takes (xpf, xpd)
    auto decide = [&](uint32_t f, float tf, uint32_t id, int pm, float xpf, double xpd) -> uint32_t {
      const bool pf = (int)f == pm;
      const float xf = pf ? xpf : xs[f];
      uint32_t right = xf > tf;
      if (xf == tf || xf != xf) {  // float tie: decide in fp64 (S5)
        const double xd = pf ? xpd : __ldg(xg + (int64_t)f * g.ldx);
        right = !(xd <= __ldg(&n16[id].v));
      }
      return right;
    };
    auto dec_k = [&](const ulonglong4& G, int pm, float xpf, double xpd) -> uint32_t {
      return decide((uint32_t)(G.x >> 32) & 0xffu, __uint_as_float((uint32_t)G.x), (uint32_t)(G.w >> 32), pm, xpf, xpd);
    };
    auto dec_c = [&](const ulonglong4& G, uint32_t r0, int pm, float xpf, double xpd) -> uint32_t {
      const unsigned long long c = r0 ? G.z : G.y;
      const uint32_t cw = (uint32_t)(c >> 32);
      return decide(cw & 0xffu, __uint_as_float((uint32_t)c), (uint32_t)(G.w >> 32) + (cw >> 8) + r0, pm, xpf, xpd);
    };
    // the grandchild slot after decisions r0, r1 (G32_LEAF set if it holds a leaf value)
    auto next_slot = [&](const ulonglong4& G, uint32_t r0, uint32_t r1) -> uint32_t {
      const uint32_t w0 = (uint32_t)(G.x >> 32);
      const uint32_t ci = 2u * (r0 & ~(w0 >> 8) & 1u) + r1;
      return ((uint32_t)G.w + ci) | (((w0 >> (10 + ci)) & 1u) ? G32_LEAF : 0u);
    };
    auto child_leaf = [&](const ulonglong4& G, uint32_t r0) -> bool { return ((uint32_t)(G.x >> 32) >> (8 + r0)) & 1u; };
    // original walk
    double f0v;
    if (rw & ROOT_LEAF) {
      f0v = __longlong_as_double((long long)ldg256(G32 + root).x);
    } else {
      ulonglong4 G = ldg256(G32 + root);
      for (;;) {
        const uint32_t r0 = dec_k(G, -1, 0.f, 0.0);
        if (child_leaf(G, r0)) {
          f0v = __longlong_as_double((long long)(r0 ? G.z : G.y));
          break;
        }
        const uint32_t ns = next_slot(G, r0, dec_c(G, r0, -1, 0.f, 0.0));
        const ulonglong4 Gn = ldg256(G32 + (ns & ~G32_LEAF));
        ++nld;
        if (ns & G32_LEAF) {
          f0v = __longlong_as_double((long long)Gn.x);
          break;
        }
        G = Gn;
      }
    }
    const double d0 = yr - f0v;
    err0 = d0 * d0;
    atomicAdd(&g.oob_sum[r], f0v);
    atomicAdd(&g.oob_cnt[r], 1);
    // permuted walks from the first occurrence of each predictor on the path, IL at a time
    if (!(rw & ROOT_LEAF)) {
      uint64_t seen = 0;
      ulonglong4 G = ldg256(G32 + root);
      uint32_t sub = 0, r0c = 0;  // cursor: at the group's node k (sub 0) or at its chosen child r0c (sub 1)
      bool at_leaf = false;
      for (;;) {
        int cnt = 0;
        int qm[IL];
        ulonglong4 qG[IL];
        uint32_t qs[IL];  // 0: start at the group's node k; 1 | r0 << 1: start at its child r0
#pragma unroll
        for (int u = 0; u < IL; ++u) qs[u] = 0;
        while (!at_leaf && cnt < IL) {
          const uint32_t m = sub == 0 ? ((uint32_t)(G.x >> 32) & 0xffu) : ((uint32_t)((r0c ? G.z : G.y) >> 32) & 0xffu);
          if (!((seen >> m) & 1ull)) {
            seen |= 1ull << m;
#pragma unroll
            for (int u = 0; u < IL; ++u)
              if (u == cnt) {
                qm[u] = (int)m;
                qG[u] = G;
                qs[u] = sub ? (1u | (r0c << 1)) : 0u;
              }
            ++cnt;
          }
          if (sub == 0) {
            r0c = dec_k(G, -1, 0.f, 0.0);
            if (child_leaf(G, r0c)) at_leaf = true;
            else sub = 1;
          } else {
            const uint32_t ns = next_slot(G, r0c, dec_c(G, r0c, -1, 0.f, 0.0));
            if (ns & G32_LEAF) {
              at_leaf = true;
            } else {
              G = ldg256(G32 + ns);
              ++nld;
              sub = 0;
            }
          }
        }
        if (cnt == 0) break;
        nrw += cnt;
        double xm[IL];
        float xmf[IL];
        bool live[IL], lpend[IL];
#pragma unroll
        for (int u = 0; u < IL; ++u) {
          live[u] = u < cnt;
          lpend[u] = false;
          xm[u] = 0.0;
          if (live[u]) {
            const int64_t pa = __ldg(g.perm + ((int64_t)b * g.p + qm[u]) * g.n + a);
            xm[u] = __ldg(g.X + (int64_t)qm[u] * g.ldx + Ob[pa]);
          } else {
            qm[u] = -1;
          }
          xmf[u] = __double2float_rn(xm[u]);
        }
        double val[IL];
        bool any = true;
        while (any) {
          any = false;
#pragma unroll
          for (int u = 0; u < IL; ++u)
            if (live[u]) {
              const ulonglong4 Gu = qG[u];
              if (lpend[u]) {  // the slot just loaded is a leaf
                val[u] = __longlong_as_double((long long)Gu.x);
                live[u] = false;
                continue;
              }
              const uint32_t r0 = (qs[u] & 1u) ? (qs[u] >> 1) : dec_k(Gu, qm[u], xmf[u], xm[u]);
              if (child_leaf(Gu, r0)) {
                val[u] = __longlong_as_double((long long)(r0 ? Gu.z : Gu.y));
                live[u] = false;
                continue;
              }
              const uint32_t ns = next_slot(Gu, r0, dec_c(Gu, r0, qm[u], xmf[u], xm[u]));
              qG[u] = ldg256(G32 + (ns & ~G32_LEAF));
              ++nld;
              qs[u] = 0;
              lpend[u] = (ns & G32_LEAF) != 0;
              any = true;
            }
        }
#pragma unroll
        for (int u = 0; u < IL; ++u)
          if (u < cnt) {
            const double d1 = yr - val[u];
            const double diff = d1 * d1 - err0;
            if (diff != 0.0) atomicAdd(&sacc[qm[u]], diff);
          }
      }
    }
    if (g3.prof) {  // one atomic pair per warp
      const unsigned act_m = __activemask();
      const uint32_t wl = __reduce_add_sync(act_m, nld), wr = __reduce_add_sync(act_m, nrw);
      if ((threadIdx.x & 31) == __ffs(act_m) - 1) {
        atomicAdd(&g3.prof[0], (unsigned long long)wl);
        atomicAdd(&g3.prof[1], (unsigned long long)wr);
      }
    }
  }
  // e_t
  for (int o = 16; o > 0; o >>= 1) err0 += __shfl_down_sync(0xffffffffu, err0, o);
  if ((threadIdx.x & 31) == 0) serr[threadIdx.x >> 5] = err0;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int j = 0; j < IPT / 32; ++j) s += serr[j];
    if (s != 0.0) atomicAdd(&g.e_t[i], s);
  }
  for (int m = threadIdx.x; m < g.p; m += IPT)
    if (sacc[m] != 0.0) atomicAdd(&g.d_slots[(int64_t)i * g.p + m], sacc[m]);
}

__global__ void k_divide(double* d_slots, const int64_t* nout_t, int32_t T, int p) {
  const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k >= (int64_t)T * p) return;
  const int64_t no = nout_t[k / p];
  d_slots[k] = no > 0 ? d_slots[k] / (double)no : 0.0;
}

// S6-S8 aggregation (one CTA; fixed reduction order -> deterministic).
__global__ void k_finalize_imp(const double* d, const double* npur, const double* oob_sum, const int32_t* oob_cnt,
                               const double* y, int64_t n, int p, int32_t T, double* o4, double* o2) {
  __shared__ double s1[NT], s2[NT];
  __shared__ long long sc[NT];
  for (int m = threadIdx.x; m < p; m += NT) {
    double raw = 0.0;
    for (int32_t t = 0; t < T; ++t) raw += d[(int64_t)t * p + m];
    raw /= (double)T;
    double v = 0.0;
    for (int32_t t = 0; t < T; ++t) {
      const double e = d[(int64_t)t * p + m] - raw;
      v += e * e;
    }
    v /= (double)T;
    const double sd = sqrt(v / (double)T);
    double np = 0.0;
    for (int32_t t = 0; t < T; ++t) np += npur[(int64_t)t * p + m];
    o4[m] = sd >= 2.220446049250313e-16 ? raw / sd : raw;
    o4[p + m] = raw;
    o4[2 * p + m] = sd;
    o4[3 * p + m] = np / (double)T;
  }
  double se = 0.0, sy = 0.0;
  long long cnt = 0;
  for (int64_t r = threadIdx.x; r < n; r += NT) {
    sy += y[r];
    if (oob_cnt[r] > 0) {
      const double e = y[r] - oob_sum[r] / (double)oob_cnt[r];
      se += e * e;
      ++cnt;
    }
  }
  s1[threadIdx.x] = se;
  s2[threadIdx.x] = sy;
  sc[threadIdx.x] = cnt;
  __syncthreads();
  for (int s = NT / 2; s > 0; s >>= 1) {
    if (threadIdx.x < s) {
      s1[threadIdx.x] += s1[threadIdx.x + s];
      s2[threadIdx.x] += s2[threadIdx.x + s];
      sc[threadIdx.x] += sc[threadIdx.x + s];
    }
    __syncthreads();
  }
  const double mse = sc[0] ? s1[0] / (double)sc[0] : 0.0;
  const double mean = s2[0] / (double)n;
  __syncthreads();
  double sv = 0.0;
  for (int64_t r = threadIdx.x; r < n; r += NT) {
    const double e = y[r] - mean;
    sv += e * e;
  }
  s1[threadIdx.x] = sv;
  __syncthreads();
  for (int s = NT / 2; s > 0; s >>= 1) {
    if (threadIdx.x < s) s1[threadIdx.x] += s1[threadIdx.x + s];
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    const double var = s1[0] / (double)n;
    o2[0] = mse;
    o2[1] = var > 0.0 ? 1.0 - mse / var : 0.0;
  }
}

}  // namespace

void perm_impl(uint64_t seed, int32_t t, int32_t m, int64_t n_o, int64_t* out, cudaStream_t s) {
  {
    KScope ks_("k_perm", s, 0.0);
    k_perm<<<(unsigned)ceil_div(n_o, NT), NT, 0, s>>>(seed, t, m, n_o, out);
  }
  BF_CUDA_CHECK(cudaGetLastError());
}

void xf_rows_impl(const double* X, int64_t ldx, int64_t n, int p, float* Xf, int xfs, cudaStream_t s) {
  if (n <= 0) return;
  KScope ks_("k_xf_rows", s, (double)n * p * 8.0 + (double)n * xfs * 4.0);
  k_xf_rows<<<dim3((unsigned)ceil_div(n, 32), (unsigned)ceil_div(xfs, 32)), dim3(32, 8), 0, s>>>(X, ldx, n, p, Xf, xfs);
  BF_CUDA_CHECK(cudaGetLastError());
}

void oob_importance_impl(const bf_forest* f, const double* X_in, int64_t ldx, const double* y_in, int64_t n, int32_t p,
                         const bf_oob_accum& acc, cudaStream_t s) {
  const int32_t T = f->info.tree_end - f->info.tree_begin;
  InStage Xs(X_in, sizeof(double) * (size_t)(ldx * (p - 1) + n), s);
  InStage ys(y_in, sizeof(double) * (size_t)n, s);
  const double* X = (const double*)Xs.dptr;
  const double* y = (const double*)ys.dptr;
  OutStage d_s(acc.d_slots, sizeof(double) * (size_t)T * p, s), np_s(acc.npur_slots, sizeof(double) * (size_t)T * p, s),
      os_s(acc.oob_sum, sizeof(double) * n, s), oc_s(acc.oob_cnt, sizeof(int32_t) * n, s),
      et_s(acc.e_t, sizeof(double) * (size_t)std::max(T, 1), s), no_s(acc.nout_t, sizeof(int64_t) * (size_t)std::max(T, 1), s);
  double* d_slots = (double*)d_s.dptr;
  double* npur = (double*)np_s.dptr;
  double* oob_sum = (double*)os_s.dptr;
  int32_t* oob_cnt = (int32_t*)oc_s.dptr;
  double* e_t = (double*)et_s.dptr;
  int64_t* nout_t = (int64_t*)no_s.dptr;
  if (T > 0) {
    BF_CUDA_CHECK(cudaMemsetAsync(d_slots, 0, sizeof(double) * (size_t)T * p, s));
    BF_CUDA_CHECK(cudaMemsetAsync(npur, 0, sizeof(double) * (size_t)T * p, s));
    BF_CUDA_CHECK(cudaMemsetAsync(e_t, 0, sizeof(double) * T, s));
  }
  BF_CUDA_CHECK(cudaMemsetAsync(oob_sum, 0, sizeof(double) * n, s));
  BF_CUDA_CHECK(cudaMemsetAsync(oob_cnt, 0, sizeof(int32_t) * n, s));
  // trees per batch: the batch's pi tables (B x p x n int32) stay under 1 GiB
  const int B = (int)std::max<int64_t>(1, std::min<int64_t>({(int64_t)T, 64, ((int64_t)1 << 28) / std::max<int64_t>(1, (int64_t)p * n)}));
  const int nchunk = (int)ceil_div(n, OCH);
  DBuf<int32_t> w((size_t)B * n, s), cnt((size_t)B * nchunk, s);
  DBuf<uint32_t> O((size_t)B * n, s);
  DBuf<int32_t> perm((size_t)B * p * n, s);
  DBuf<uint8_t> used((size_t)B * p, s);
  int hb_all = 64 - __builtin_clzll((unsigned long long)std::max<int64_t>(n - 1, 1));
  hb_all = std::max(hb_all, 2);
  hb_all += hb_all & 1;
  DBuf<uint32_t> gtab((size_t)B * p * (6u << std::min(hb_all / 2, PH_MAX)), s);
  size_t smem = sizeof(double) * ((size_t)((p + 1) & ~1) + (size_t)IPT * (size_t)(p | 1));
  static int ismax = 0;
  if (!ismax) ismax = std::min(dyn_smem_limit(k_importance<IPT>), dyn_smem_limit(k_importance<IPT_WIDE>));
  const bool wide = smem > (size_t)ismax;
  if (wide) smem = sizeof(double) * ((size_t)((p + 1) & ~1) + (size_t)IPT_WIDE * (size_t)(p | 1));
  BF_REQUIRE(smem <= (size_t)ismax, BF_ENOTIMPL, "bf_oob_importance: p too large for the shared-memory row tile");
  const char* force16 = getenv("BF_PREDICT_NODE16");  // same switch as predict: keep the Node16 walks
  const size_t smem8 = sizeof(double) * (size_t)((p + 1) & ~1) + sizeof(float) * (size_t)IPT * (size_t)(p | 1);
  static int ismax8 = 0;
  if (!ismax8) ismax8 = dyn_smem_limit(k_importance8);
  // walks on the two-level groups when the forest has them and p <= 64 (BF_PREDICT_V=2 keeps the Node8 walks)
  static int ismax32 = 0;
  if (!ismax32)
    ismax32 = std::min(std::min(dyn_smem_limit(k_importance32<2>), dyn_smem_limit(k_importance32<3>)),
                       dyn_smem_limit(k_importance32<4>));
  // permuted walks interleaved per thread (measured per 200 C4 trees: 3 -> 119 ms, 4 -> 142 ms)
  static const int il32 = getenv("BF_IMP32_ILP") ? atoi(getenv("BF_IMP32_ILP")) : 3;
  const char* pvs = getenv("BF_PREDICT_V");
  const bool want32 = p <= 64 && !(force16 && force16[0] == '1') && !(pvs && atoi(pvs) != 3);
  const ulonglong4* g32 = want32 ? g32_get(const_cast<bf_forest*>(f), s) : nullptr;
  const uint2* n8 = (force16 && force16[0] == '1') || (g32 && smem8 <= (size_t)ismax32)
                        ? nullptr : nodes8_get(const_cast<bf_forest*>(f), s);
  DBuf<unsigned long long> prof;
  if (prof_enabled()) {
    prof.alloc(2, s);
    BF_CUDA_CHECK(cudaMemsetAsync(prof.p, 0, 16, s));
  }
  DBuf<float> Xf;
  const int xfs = (p + 3) & ~3;
  for (int32_t i0 = 0; i0 < T; i0 += B) {
    const int Bc = std::min(B, T - i0);
    bootstrap_impl(f->info.seed, f->info.tree_begin + i0, Bc, n, f->info.sampsize, f->info.replace, w.p, s);
    {
      KScope ks_("k_oob_count", s, 0.0);
      k_oob_count<<<dim3(nchunk, Bc), NT, 0, s>>>(w.p, n, nchunk, cnt.p);
    }
    {
      KScope ks_("k_oob_prefix", s, 0.0);
      k_oob_prefix<<<(unsigned)ceil_div(Bc, 64), 64, 0, s>>>(cnt.p, Bc, nchunk, nout_t + i0);
    }
    {
      KScope ks_("k_oob_scatter", s, 0.0);
      k_oob_scatter<<<dim3(nchunk, Bc), NT, 0, s>>>(w.p, n, nchunk, cnt.p, O.p);
    }
    {
      KScope ks_("k_npur", s, 0.0);
      BF_CUDA_CHECK(cudaMemsetAsync(used.p, 0, (size_t)Bc * p, s));
      k_npur<<<dim3(64, Bc), NT, (sizeof(double) + sizeof(int)) * (size_t)p, s>>>(f->d_nodes, f->d_drss, f->d_tree_off,
                                                                                 i0, p, npur, used.p);
    }
    {
      static int pfs = 0;
      if (!pfs) pfs = dyn_smem_limit(k_perm_fill);
      // round tables sized for the largest possible n_o (<= n): 6 x 2^h words, h = feistel_h(n) <= PH_MAX
      int hb = 64 - __builtin_clzll((unsigned long long)std::max<int64_t>(n - 1, 1));
      hb = std::max(hb, 2);
      hb += hb & 1;
      const int hmax = std::min(hb / 2, PH_MAX);
      const int tstride = 6 << hmax;
      {
        KScope ks2_("k_ftab_fill", s, 0.0);
        k_ftab_fill<<<dim3((unsigned)ceil_div(tstride, 256), p, Bc), 256, 0, s>>>(f->info.seed, f->info.tree_begin + i0, p,
                                                                              nout_t + i0, tstride, gtab.p);
      }
      KScope ks_("k_perm_fill", s, 0.0);
      k_perm_fill<<<dim3((unsigned)std::max<int64_t>(1, std::min<int64_t>(8, ceil_div(n, 65536))), p, Bc), 512,
                    sizeof(uint32_t) * 6 * ((size_t)1 << hmax), s>>>(f->info.seed, f->info.tree_begin + i0, p, n,
                                                                     nout_t + i0, gtab.p, tstride, perm.p, used.p);
    }
    BF_CUDA_CHECK(cudaGetLastError());
    ImpArgs g;
    g.nodes = f->d_nodes;
    g.off = f->d_tree_off;
    g.X = X;
    g.ldx = ldx;
    g.y = y;
    g.n = n;
    g.p = p;
    g.seed = f->info.seed;
    g.tree_begin = f->info.tree_begin;
    g.i0 = i0;
    g.O = O.p;
    g.nout = nout_t + i0;
    g.d_slots = d_slots;
    g.oob_sum = oob_sum;
    g.oob_cnt = oob_cnt;
    g.e_t = e_t;
    g.perm = perm.p;
    // OOB rows per tree <= n; grid sized for n (CTAs past n_o exit early)
    if (g32 && smem8 <= (size_t)ismax32) {
      if (!Xf.p) {  // once per call: the row-major float copy the CTAs stage their OOB rows from
        Xf.alloc((size_t)n * xfs, s);
        xf_rows_impl(X, ldx, n, p, Xf.p, xfs, s);
      }
      Imp32Args g3;
      g3.a = g;
      g3.Xf = Xf.p;
      g3.xfs = xfs;
      g3.g32 = g32;
      g3.roots32 = f->d_g32_root;
      g3.prof = prof.p;
      KScope ks_("k_importance32", s, 0.0);
      if (il32 == 2)
        k_importance32<2><<<dim3((unsigned)ceil_div(n, IPT), Bc), IPT, smem8, s>>>(g3);
      else if (il32 == 4)
        k_importance32<4><<<dim3((unsigned)ceil_div(n, IPT), Bc), IPT, smem8, s>>>(g3);
      else
        k_importance32<3><<<dim3((unsigned)ceil_div(n, IPT), Bc), IPT, smem8, s>>>(g3);
    } else if (n8 && smem8 <= (size_t)ismax8) {
      if (!Xf.p) {  // once per call: the row-major float copy the CTAs stage their OOB rows from
        Xf.alloc((size_t)n * xfs, s);
        xf_rows_impl(X, ldx, n, p, Xf.p, xfs, s);
      }
      Imp8Args g8;
      g8.a = g;
      g8.Xf = Xf.p;
      g8.xfs = xfs;
      g8.nodes8 = n8;
      g8.roots8 = f->d_roots8;
      g8.prof = prof.p;
      KScope ks_("k_importance8", s, 0.0);
      k_importance8<<<dim3((unsigned)ceil_div(n, IPT), Bc), IPT, smem8, s>>>(g8);
    } else {
      KScope ks_("k_importance", s, 0.0);
      if (wide)
        k_importance<IPT_WIDE><<<dim3((unsigned)ceil_div(n, IPT_WIDE), Bc), IPT_WIDE, smem, s>>>(g);
      else
        k_importance<IPT><<<dim3((unsigned)ceil_div(n, IPT), Bc), IPT, smem, s>>>(g);
    }
    BF_CUDA_CHECK(cudaGetLastError());
  }
  if (prof.p && T > 0) {  // algorithmic bytes of k_importance8
    unsigned long long hp[2] = {0, 0};
    std::vector<int64_t> hno(T);
    BF_CUDA_CHECK(cudaMemcpyAsync(hp, prof.p, 16, cudaMemcpyDeviceToHost, s));
    BF_CUDA_CHECK(cudaMemcpyAsync(hno.data(), nout_t, sizeof(int64_t) * T, cudaMemcpyDeviceToHost, s));
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
    double units = 0.0;
    for (int64_t v : hno) units += (double)v;
    // per (tree, OOB row): float row gather 4p + y 8 + O index 4 + oob sum/count 12; per re-walk: pi 4 + x 8;
    // per node load 8 (compact nodes)
    const bool used32 = g32 && smem8 <= (size_t)ismax32;
    prof_add_bytes(used32 ? "k_importance32" : "k_importance8",
                   units * (4.0 * p + 24.0) + (double)hp[1] * 12.0 + (double)hp[0] * (used32 ? 32.0 : 8.0));
    prof_add_bytes("importance_node_loads", (double)hp[0]);
    prof_add_bytes("importance_rewalks", (double)hp[1]);
  }
  if (T > 0) {
    {
      KScope ks_("k_divide", s, 0.0);
      k_divide<<<(unsigned)ceil_div((int64_t)T * p, NT), NT, 0, s>>>(d_slots, nout_t, T, p);
    }
    BF_CUDA_CHECK(cudaGetLastError());
  }
  d_s.finish(s);
  np_s.finish(s);
  os_s.finish(s);
  oc_s.finish(s);
  et_s.finish(s);
  no_s.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

void importance_finalize_impl(const double* d_slots, const double* npur_slots, const double* oob_sum,
                              const int32_t* oob_cnt, const double* y, int64_t n, int32_t p, int32_t ntree,
                              double* o4, double* o2, cudaStream_t s) {
  {
    KScope ks_("k_finalize_imp", s, 0.0);
    k_finalize_imp<<<1, NT, 0, s>>>(d_slots, npur_slots, oob_sum, oob_cnt, y, n, p, ntree, o4, o2);
  }
  BF_CUDA_CHECK(cudaGetLastError());
}

}  // namespace bf
