// predict.cu -- batched forest prediction (P:95 step 3, S5).
//
// One thread per query row; a CTA stages its rows' predictors in shared
// memory row-major (coalesced column loads), then every thread walks all the
// forest's trees in tree order (16-byte node loads through the read-only
// path) and sums the leaf values in fp64.  All CTAs advance through the trees
// in the same order, so the trees being walked at any moment stay L2-resident.
#include <algorithm>
#include <cstdlib>

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
  if (visits) {  // one atomic per warp
    const unsigned act = __activemask();
    const unsigned long long wv = __reduce_add_sync(act, (uint32_t)nv);
    if ((threadIdx.x & 31) == __ffs(act) - 1) atomicAdd(visits, wv);
  }
  yhat_sum[rr] = acc;
  if (last && yhat) yhat[rr] = acc * inv_t;
}

// ------------------------------------------------------------------ compact 8-byte traversal nodes
// Node8 (built once per forest from Node16 by k_pack8):
//   internal: word0 = float bits of RN_f32(thr); word1 = LL<<31 | RL<<30 | feature<<22 | rel
//             (LL/RL: the left/right child is a leaf; rel = left child's id - this node's id >= 1, so the
//             children of global node g are g + rel and g + rel + 1)
//   leaf:     the 8 bytes are the fp64 leaf value (a walk lands on a leaf only through its parent's LL/RL
//             bit, or at the root of a single-node tree, flagged in the tree's root word).
// The comparison x <= thr of S5 is decided on floats where that is exact: rounding to float is monotone, so
// RN_f32(x) < RN_f32(thr) implies x < thr and RN_f32(x) > RN_f32(thr) implies x > thr; only
// RN_f32(x) == RN_f32(thr) (or NaN) falls back to the fp64 x (global X) and the fp64 thr (Node16).  The walk
// therefore takes exactly the S5 path, with half the node bytes and half the shared-memory row tile.

__global__ void k_pack8(const Node16* __restrict__ nodes, const int64_t* __restrict__ off, uint2* __restrict__ out,
                        uint32_t* __restrict__ roots, int* __restrict__ bad) {
  const int32_t t = blockIdx.y;
  const int64_t lo = off[t], hi = off[t + 1];
  if (blockIdx.x == 0 && threadIdx.x == 0) roots[t] = (uint32_t)lo | (hi - lo == 1 ? ROOT_LEAF : 0u);
  for (int64_t k = lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < hi; k += (int64_t)gridDim.x * blockDim.x) {
    const Node16 nd = nodes[k];
    uint2 o;
    if (nd.feature < 0) {
      const unsigned long long b = (unsigned long long)__double_as_longlong(nd.v);
      o.x = (uint32_t)b;
      o.y = (uint32_t)(b >> 32);
    } else {
      const int64_t rel = (int64_t)nd.left - (k - lo);
      if (rel < 1 || rel >= (1ll << N8_REL_BITS) || lo + nd.left + 1 >= hi) {
        *bad = 1;  // children not after their parent: the forest keeps the Node16 path
        o = make_uint2(0u, 0u);
      } else {
        const uint32_t ll = nodes[lo + nd.left].feature < 0, rl = nodes[lo + nd.left + 1].feature < 0;
        o.x = __float_as_uint(__double2float_rn(nd.v));
        o.y = (ll << 31) | (rl << 30) | ((uint32_t)nd.feature << N8_REL_BITS) | (uint32_t)rel;
      }
    }
    out[k] = o;
  }
}


constexpr int PT8 = 128;  // rows per CTA
constexpr int S8 = 8;     // walks in flight per thread (a finished slot restarts with the block's next tree;
                          // measured: 12 or 16 slots lower occupancy and run slower)

// Trees [t_begin, t_end) of one tree block for every row of the CTA's tile (a block is a few trees that stay
// L2-resident while all CTAs walk it).  Each thread keeps S8 walks in flight, a slot being (global node id,
// node word); a slot that reaches a leaf adds the value and restarts at the block's next tree (a fixed order
// per row: deterministic sums).  PROF counts node loads and fp64 fallbacks (profile mode only).
template <bool PROF>
__global__ void __launch_bounds__(PT8, 6) k_predict8(const uint2* __restrict__ nodes8, const Node16* __restrict__ nodes16,
                                                     const uint32_t* __restrict__ roots, int32_t t_begin, int32_t t_end,
                                                     int first, int last, const double* __restrict__ Xq, int64_t ldq,
                                                     int64_t m, int p, double* yhat_sum, double* yhat, double inv_t,
                                                     unsigned long long* visits) {
  extern __shared__ float sxf[];  // PT8 x (p|1), row-major
  const int stride = p | 1;
  const int64_t r0 = (int64_t)blockIdx.x * PT8;
  const int rows = (int)(m - r0 < PT8 ? m - r0 : PT8);
  {  // stage the tile as floats: 8 column loads in flight per thread
    const int r = threadIdx.x;
    const bool ok = r < rows;
    const double* src = Xq + r0 + (ok ? r : 0);
    for (int f0 = 0; f0 < p; f0 += 8) {
      double v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) v[u] = (f0 + u < p) ? __ldcs(src + (int64_t)(f0 + u) * ldq) : 0.0;
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (f0 + u < p && ok) sxf[r * stride + f0 + u] = __double2float_rn(v[u]);
    }
  }
  __syncthreads();
  if ((int)threadIdx.x >= rows) return;
  const float* xs = sxf + threadIdx.x * stride;
  const int64_t rr = r0 + threadIdx.x;
  const double* xg = Xq + rr;
  double acc = first ? 0.0 : yhat_sum[rr];
  uint32_t nv = 0, nfb = 0;
  uint32_t gid[S8];  // global node id of the slot's current node; ~0u = idle
  uint2 nd[S8];
  int32_t tnext = t_begin;
  // next non-trivial tree of the block into slot u (single-node trees add their value at once)
  auto start = [&](int u) {
    gid[u] = ~0u;
    while (tnext < t_end) {
      const uint32_t rw = __ldg(roots + tnext++);
      const uint2 rn = __ldg(nodes8 + (rw & ~ROOT_LEAF));
      if (PROF) ++nv;
      if (rw & ROOT_LEAF) {
        acc += leaf8(rn);
        continue;
      }
      gid[u] = rw;
      nd[u] = rn;
      break;
    }
  };
#pragma unroll
  for (int u = 0; u < S8; ++u) start(u);
  bool any = true;
  while (any) {
    any = false;
#pragma unroll
    for (int u = 0; u < S8; ++u) {
      if (gid[u] == ~0u) continue;
      any = true;
      const uint2 w = nd[u];
      const uint32_t f = (w.y >> N8_REL_BITS) & ((1u << N8_FEAT_BITS) - 1u);
      const float xf = xs[f], tf = __uint_as_float(w.x);
      uint32_t right = xf > tf;
      if (xf == tf || xf != xf) {  // float tie (or NaN): decide in fp64 (S5)
        right = !(__ldg(xg + (int64_t)f * ldq) <= __ldg(&nodes16[gid[u]].v));
        if (PROF) ++nfb;
      }
      const uint32_t c = gid[u] + (w.y & ((1u << N8_REL_BITS) - 1u)) + right;
      const uint2 ch = __ldg(nodes8 + c);
      if (PROF) ++nv;
      if ((w.y >> (31 - right)) & 1u) {
        acc += leaf8(ch);
        start(u);
      } else {
        gid[u] = c;
        nd[u] = ch;
      }
    }
  }
  if (PROF) {  // one atomic per warp (per-thread atomics on one address would serialise in L2)
    const unsigned act = __activemask();
    const uint32_t wv = __reduce_add_sync(act, nv), wf = __reduce_add_sync(act, nfb);
    if ((threadIdx.x & 31) == __ffs(act) - 1) {
      atomicAdd(visits, (unsigned long long)wv);
      atomicAdd(visits + 1, (unsigned long long)wf);
    }
  }
  yhat_sum[rr] = acc;
  if (last && yhat) yhat[rr] = acc * inv_t;
}

// k_predict8 with the tree block's root words and root nodes staged in shared memory (a slot restarts from
// shared memory, not with two dependent global loads) and the float-tie fp64 fallback out of line (no
// predicated global loads on the common path).  Used for blocks of <= RT8 trees (BF_PREDICT_V=1 restores
// k_predict8).
constexpr int RT8 = 64;
__device__ __noinline__ uint32_t tie_right_fp64(const double* xg, int64_t ldq, uint32_t f, const Node16* n16,
                                                uint32_t gid) {
  return !(__ldg(xg + (int64_t)f * ldq) <= __ldg(&n16[gid].v));
}

template <bool PROF, int NS>
__global__ void __launch_bounds__(PT8, 6) k_predict8s(const uint2* __restrict__ nodes8, const Node16* __restrict__ nodes16,
                                                      const uint32_t* __restrict__ roots, int32_t t_begin, int32_t t_end,
                                                      int first, int last, const double* __restrict__ Xq, int64_t ldq,
                                                      int64_t m, int p, double* yhat_sum, double* yhat, double inv_t,
                                                      unsigned long long* visits) {
  extern __shared__ float sxf[];  // PT8 x (p|1), row-major
  __shared__ uint32_t s_rw[RT8];
  __shared__ uint2 s_rn[RT8];
  const int stride = p | 1;
  const int64_t r0 = (int64_t)blockIdx.x * PT8;
  const int rows = (int)(m - r0 < PT8 ? m - r0 : PT8);
  const int nt = t_end - t_begin;
  if ((int)threadIdx.x < nt) {
    const uint32_t rw = __ldg(roots + t_begin + threadIdx.x);
    s_rw[threadIdx.x] = rw;
    s_rn[threadIdx.x] = __ldg(nodes8 + (rw & ~ROOT_LEAF));
  }
  {  // stage the tile as floats: 8 column loads in flight per thread
    const int r = threadIdx.x;
    const bool ok = r < rows;
    const double* src = Xq + r0 + (ok ? r : 0);
    for (int f0 = 0; f0 < p; f0 += 8) {
      double v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) v[u] = (f0 + u < p) ? __ldcs(src + (int64_t)(f0 + u) * ldq) : 0.0;
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (f0 + u < p && ok) sxf[r * stride + f0 + u] = __double2float_rn(v[u]);
    }
  }
  __syncthreads();
  if ((int)threadIdx.x >= rows) return;
  const float* xs = sxf + threadIdx.x * stride;
  const int64_t rr = r0 + threadIdx.x;
  const double* xg = Xq + rr;
  double acc = first ? 0.0 : yhat_sum[rr];
  uint32_t nv = 0, nfb = 0;
  uint32_t gid[NS];
  uint2 nd[NS];
  int tnext = 0;
  int nact = 0;
  auto start = [&](int u) {
    gid[u] = ~0u;
    while (tnext < nt) {
      const uint32_t rw = s_rw[tnext];
      const uint2 rn = s_rn[tnext];
      ++tnext;
      if (PROF) ++nv;
      if (rw & ROOT_LEAF) {
        acc += leaf8(rn);
        continue;
      }
      gid[u] = rw;
      nd[u] = rn;
      ++nact;
      break;
    }
  };
#pragma unroll
  for (int u = 0; u < NS; ++u) start(u);
  while (nact > 0) {
#pragma unroll
    for (int u = 0; u < NS; ++u) {
      if (gid[u] == ~0u) continue;
      const uint2 w = nd[u];
      const uint32_t f = (w.y >> N8_REL_BITS) & ((1u << N8_FEAT_BITS) - 1u);
      const float xf = xs[f], tf = __uint_as_float(w.x);
      uint32_t right = xf > tf;
      if (__builtin_expect(xf == tf || xf != xf, 0)) {  // float tie (or NaN): decide in fp64 (S5)
        right = tie_right_fp64(xg, ldq, f, nodes16, gid[u]);
        if (PROF) ++nfb;
      }
      const uint32_t c = gid[u] + (w.y & ((1u << N8_REL_BITS) - 1u)) + right;
      const uint2 ch = __ldg(nodes8 + c);
      if (PROF) ++nv;
      if ((w.y >> (31 - right)) & 1u) {
        acc += leaf8(ch);
        --nact;
        start(u);
      } else {
        gid[u] = c;
        nd[u] = ch;
      }
    }
  }
  if (PROF) {
    const unsigned act = __activemask();
    const uint32_t wv = __reduce_add_sync(act, nv), wf = __reduce_add_sync(act, nfb);
    if ((threadIdx.x & 31) == __ffs(act) - 1) {
      atomicAdd(visits, (unsigned long long)wv);
      atomicAdd(visits + 1, (unsigned long long)wf);
    }
  }
  yhat_sum[rr] = acc;
  if (last && yhat) yhat[rr] = acc * inv_t;
}


// ------------------------------------------------------------------ two-level 32-byte groups (G32)
// Every node at even depth owns a slot of 32 bytes.  For an internal node k (children L, R = L + 1):
//   q0 = {float RN_f32(thr_k), feature_k | LL<<8 | RL<<9 | GL<<10 (4 bits: grandchild slot is a leaf)}
//   q1 = L: leaf -> its fp64 value; internal -> {float RN_f32(thr_L), feature_L | rel<<8}  (rel = id(L) - id(k))
//   q2 = R: likewise, rel the same (id(R) = id(k) + rel + 1)
//   q3 = {first grandchild slot (global), id(k) (global Node16 index, for the fp64 tie fallback)}
// The grandchildren (children of L if L is internal, then children of R if R is internal) occupy consecutive
// slots from q3.lo; a grandchild that is a leaf holds its fp64 value in q0.  One 256-bit load per group decides
// two levels of a walk (S5: x <= thr goes left), with the same float-then-fp64 comparison as Node8.
// Slots: depth parity by pointer jumping over parent links, then per group the number of grandchild slots,
// one exclusive scan (the root of every tree takes one extra slot first), and the slots written top-down.

__global__ void k_g32_parent(const Node16* __restrict__ nodes, const int64_t* __restrict__ off, int32_t* anc,
                             uint8_t* bit) {
  const int32_t t = blockIdx.y;
  const int64_t lo = off[t], hi = off[t + 1];
  for (int64_t k = lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < hi; k += (int64_t)gridDim.x * blockDim.x) {
    if (k == lo) {
      anc[k] = -1;
      bit[k] = 0;
    }
    const Node16 nd = nodes[k];
    if (nd.feature >= 0) {
      const int64_t c = lo + nd.left;
      anc[c] = (int32_t)k;
      anc[c + 1] = (int32_t)k;
      bit[c] = 1;
      bit[c + 1] = 1;
    }
  }
}

// one pointer-jumping round: bit = parity of the distance to anc; anc moves twice as far up
__global__ void k_g32_jump(const int32_t* __restrict__ anc, const uint8_t* __restrict__ bit, int32_t* anc2,
                           uint8_t* bit2, int64_t total, int* more) {
  const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k >= total) return;
  const int32_t a = anc[k];
  if (a < 0) {
    anc2[k] = -1;
    bit2[k] = bit[k];
    return;
  }
  const int32_t aa = anc[a];
  anc2[k] = aa;
  bit2[k] = bit[k] ^ bit[a];
  if (aa >= 0) *more = 1;
}

// grandchild slots of every group (even-depth internal node), plus the root's own slot
__global__ void k_g32_count(const Node16* __restrict__ nodes, const int64_t* __restrict__ off,
                            const uint8_t* __restrict__ bit, uint32_t* cnt) {
  const int32_t t = blockIdx.y;
  const int64_t lo = off[t], hi = off[t + 1];
  for (int64_t k = lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < hi; k += (int64_t)gridDim.x * blockDim.x) {
    uint32_t c = k == lo;
    const Node16 nd = nodes[k];
    if (bit[k] == 0 && nd.feature >= 0) {
      const int64_t l = lo + nd.left;
      c += 2u * (nodes[l].feature >= 0) + 2u * (nodes[l + 1].feature >= 0);
    }
    cnt[k] = c;
  }
}

__global__ void k_g32_slots(const Node16* __restrict__ nodes, const int64_t* __restrict__ off,
                            const uint8_t* __restrict__ bit, const uint32_t* __restrict__ ex, uint32_t* slot,
                            int64_t* tree_slot) {
  const int32_t t = blockIdx.y;
  const int64_t lo = off[t], hi = off[t + 1];
  for (int64_t k = lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < hi; k += (int64_t)gridDim.x * blockDim.x) {
    if (k == lo) {
      slot[k] = ex[k];
      tree_slot[t] = ex[k];
    }
    const Node16 nd = nodes[k];
    if (bit[k] != 0 || nd.feature < 0) continue;
    uint32_t b = ex[k] + (k == lo);
    const int64_t l = lo + nd.left;
#pragma unroll
    for (int c = 0; c < 2; ++c) {
      const Node16 ch = nodes[l + c];
      if (ch.feature >= 0) {
        slot[lo + ch.left] = b++;
        slot[lo + ch.left + 1] = b++;
      }
    }
  }
}

__device__ __forceinline__ unsigned long long g32_child(const Node16& ch, uint32_t rel, int* bad) {
  if (ch.feature < 0) return (unsigned long long)__double_as_longlong(ch.v);
  return (unsigned long long)__float_as_uint(__double2float_rn(ch.v)) |
         ((unsigned long long)((uint32_t)ch.feature | (rel << 8)) << 32);
}

__global__ void k_g32_emit(const Node16* __restrict__ nodes, const int64_t* __restrict__ off,
                           const uint8_t* __restrict__ bit, const uint32_t* __restrict__ ex,
                           const uint32_t* __restrict__ slot, ulonglong4* __restrict__ g32, uint32_t* __restrict__ roots,
                           int* bad) {
  const int32_t t = blockIdx.y;
  const int64_t lo = off[t], hi = off[t + 1];
  if (blockIdx.x == 0 && threadIdx.x == 0) roots[t] = slot[lo] | (nodes[lo].feature < 0 ? ROOT_LEAF : 0u);
  for (int64_t k = lo + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < hi; k += (int64_t)gridDim.x * blockDim.x) {
    if (bit[k] != 0) continue;
    const Node16 nd = nodes[k];
    ulonglong4 G = make_ulonglong4(0ull, 0ull, 0ull, 0ull);
    if (nd.feature < 0) {
      G.x = (unsigned long long)__double_as_longlong(nd.v);
    } else {
      const int64_t l = lo + nd.left;
      const int64_t rel = l - k;
      if (rel < 1 || rel >= (1ll << 24) || nd.feature >= 256) {
        *bad = 1;
        continue;
      }
      const Node16 L = nodes[l], R = nodes[l + 1];
      uint32_t gl = 0, gi = 0;
      if (L.feature >= 0) {
        gl |= (uint32_t)(nodes[lo + L.left].feature < 0) << gi;
        gl |= (uint32_t)(nodes[lo + L.left + 1].feature < 0) << (gi + 1);
        gi += 2;
        if (L.feature >= 256) *bad = 1;
      }
      if (R.feature >= 0) {
        gl |= (uint32_t)(nodes[lo + R.left].feature < 0) << gi;
        gl |= (uint32_t)(nodes[lo + R.left + 1].feature < 0) << (gi + 1);
        if (R.feature >= 256) *bad = 1;
      }
      const uint32_t w0 = (uint32_t)nd.feature | ((uint32_t)(L.feature < 0) << 8) | ((uint32_t)(R.feature < 0) << 9) |
                          (gl << 10);
      G.x = (unsigned long long)__float_as_uint(__double2float_rn(nd.v)) | ((unsigned long long)w0 << 32);
      G.y = g32_child(L, (uint32_t)rel, bad);
      G.z = g32_child(R, (uint32_t)rel, bad);
      G.w = (unsigned long long)(ex[k] + (k == lo)) | ((unsigned long long)(uint32_t)k << 32);
    }
    g32[slot[k]] = G;
  }
}


// k_predict8s on G32 groups: a slot (walk in flight) holds the 32 bytes of its current group; per step it
// decides the group's node and the chosen child, then loads the grandchild's slot (a leaf slot ends the walk
// one load later).  Trees [t_begin, t_end) of one block, rows staged as floats exactly as in k_predict8s.
template <bool PROF, int NS>
__global__ void __launch_bounds__(PT8) k_predict32(const ulonglong4* __restrict__ g32, const Node16* __restrict__ nodes16,
                                                   const uint32_t* __restrict__ roots, int32_t t_begin, int32_t t_end,
                                                   int first, int last, const double* __restrict__ Xq, int64_t ldq,
                                                   const float* __restrict__ Xqf, int xfs,
                                                   int64_t m, int p, double* yhat_sum, double* yhat, double inv_t,
                                                   unsigned long long* visits) {
  extern __shared__ float sxf[];  // PT8 x (p|1), row-major
  __shared__ uint32_t s_rw[RT8];
  __shared__ ulonglong4 s_rn[RT8];
  const int stride = p | 1;
  const int64_t r0 = (int64_t)blockIdx.x * PT8;
  const int rows = (int)(m - r0 < PT8 ? m - r0 : PT8);
  const int nt = t_end - t_begin;
  if ((int)threadIdx.x < nt) {
    const uint32_t rw = __ldg(roots + t_begin + threadIdx.x);
    s_rw[threadIdx.x] = rw;
    s_rn[threadIdx.x] = ldg256(g32 + (rw & ~ROOT_LEAF));
  }
  if (Xqf) {  // stage the tile from the row-major float copy: the row's 4 p bytes as 16-byte loads, 8 in flight
    const int r = threadIdx.x;
    if (r < rows) {
      const float4* src = reinterpret_cast<const float4*>(Xqf + (r0 + r) * (int64_t)xfs);
      float* xs = sxf + r * stride;
      const int nq = (p + 3) >> 2;
      for (int q0 = 0; q0 < nq; q0 += 8) {
        float4 v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = (q0 + u < nq) ? __ldcs(src + q0 + u) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const int f = 4 * (q0 + u);
          if (f < p) xs[f] = v[u].x;
          if (f + 1 < p) xs[f + 1] = v[u].y;
          if (f + 2 < p) xs[f + 2] = v[u].z;
          if (f + 3 < p) xs[f + 3] = v[u].w;
        }
      }
    }
  } else {  // stage the tile as floats: 8 column loads in flight per thread
    const int r = threadIdx.x;
    const bool ok = r < rows;
    const double* src = Xq + r0 + (ok ? r : 0);
    for (int f0 = 0; f0 < p; f0 += 8) {
      double v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) v[u] = (f0 + u < p) ? __ldcs(src + (int64_t)(f0 + u) * ldq) : 0.0;
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (f0 + u < p && ok) sxf[r * stride + f0 + u] = __double2float_rn(v[u]);
    }
  }
  __syncthreads();
  if ((int)threadIdx.x >= rows) return;
  const float* xs = sxf + threadIdx.x * stride;
  const int64_t rr = r0 + threadIdx.x;
  const double* xg = Xq + rr;
  double acc = first ? 0.0 : yhat_sum[rr];
  uint32_t nv = 0, nfb = 0;
  uint32_t gs[NS];
  ulonglong4 nd[NS];
  int tnext = 0;
  int nact = 0;
  auto start = [&](int u) {
    gs[u] = ~0u;
    while (tnext < nt) {
      const uint32_t rw = s_rw[tnext];
      const ulonglong4 rn = s_rn[tnext];
      ++tnext;
      if (PROF) ++nv;
      if (rw & ROOT_LEAF) {
        acc += __longlong_as_double((long long)rn.x);
        continue;
      }
      gs[u] = rw;
      nd[u] = rn;
      ++nact;
      break;
    }
  };
#pragma unroll
  for (int u = 0; u < NS; ++u) start(u);
  while (nact > 0) {
#pragma unroll
    for (int u = 0; u < NS; ++u) {
      if (gs[u] == ~0u) continue;
      const ulonglong4 G = nd[u];
      if (gs[u] & G32_LEAF) {
        acc += __longlong_as_double((long long)G.x);
        --nact;
        start(u);
        continue;
      }
      const uint32_t w0 = (uint32_t)(G.x >> 32);
      const uint32_t f0 = w0 & 0xffu;
      const float xf0 = xs[f0], tf0 = __uint_as_float((uint32_t)G.x);
      uint32_t right = xf0 > tf0;
      if (__builtin_expect(xf0 == tf0 || xf0 != xf0, 0)) {  // float tie (or NaN): decide in fp64 (S5)
        right = tie_right_fp64(xg, ldq, f0, nodes16, (uint32_t)(G.w >> 32));
        if (PROF) ++nfb;
      }
      const unsigned long long c = right ? G.z : G.y;
      if ((w0 >> (8 + right)) & 1u) {  // the chosen child is a leaf: c is its value
        acc += __longlong_as_double((long long)c);
        --nact;
        start(u);
        continue;
      }
      const uint32_t cw = (uint32_t)(c >> 32);
      const uint32_t f1 = cw & 0xffu;
      const float xf1 = xs[f1], tf1 = __uint_as_float((uint32_t)c);
      uint32_t r1 = xf1 > tf1;
      if (__builtin_expect(xf1 == tf1 || xf1 != xf1, 0)) {
        r1 = tie_right_fp64(xg, ldq, f1, nodes16, (uint32_t)(G.w >> 32) + (cw >> 8) + right);
        if (PROF) ++nfb;
      }
      const uint32_t ci = 2u * (right & ~(w0 >> 8) & 1u) + r1;  // going right past an internal L: skip its 2
      uint32_t ns = (uint32_t)G.w + ci;
      nd[u] = ldg256(g32 + ns);
      if (PROF) ++nv;
      if ((w0 >> (10 + ci)) & 1u) ns |= G32_LEAF;
      gs[u] = ns;
    }
  }
  if (PROF) {
    const unsigned act = __activemask();
    const uint32_t wv = __reduce_add_sync(act, nv), wf = __reduce_add_sync(act, nfb);
    if ((threadIdx.x & 31) == __ffs(act) - 1) {
      atomicAdd(visits, (unsigned long long)wv);
      atomicAdd(visits + 1, (unsigned long long)wf);
    }
  }
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
  if (visits) {  // one atomic per warp
    const unsigned act = __activemask();
    const unsigned long long wv = __reduce_add_sync(act, (uint32_t)nv);
    if ((threadIdx.x & 31) == __ffs(act) - 1) atomicAdd(visits, wv);
  }
  if (yhat_sum) yhat_sum[r] = acc;
  if (yhat) yhat[r] = acc * inv_t;
}

// ------------------------------------------------------------------ partial dependence
// P:130 ("the partial dependence plot, shows how the response changes as a
// predictor ... change(s)"); readings R23 (grid) and R24 (definition):
//   pd_sum[g] = sum_i sum_t f_t(x_i with x_im := v_g).
// CTA = (tile of PT training rows, grid point g): the tile is staged like the
// predict tile, column m is overwritten with v_g, the rows walk the tree
// block (8 walks in flight per thread), the CTA reduces its rows' sums and
// adds one value to pd_sum[g] (fp64 atomics: order-free up to rounding, R22).
__global__ void __launch_bounds__(PT) k_pdep(const Node16* __restrict__ nodes, const int64_t* __restrict__ off,
                                             int32_t t_begin, int32_t t_end, const double* __restrict__ X, int64_t ldx,
                                             int64_t n, int p, int mcol, const double* __restrict__ grid,
                                             double* pd_sum) {
  extern __shared__ double sx[];
  __shared__ double sred[PT / 32];
  const int stride = p | 1;
  const int64_t r0 = (int64_t)blockIdx.x * PT;
  const int rows = (int)(n - r0 < PT ? n - r0 : PT);
  const double vg = grid[blockIdx.y];
  {
    const int r = threadIdx.x;
    const bool ok = r < rows;
    const double* src = X + r0 + (ok ? r : 0);
    for (int f0 = 0; f0 < p; f0 += 16) {
      double v[16];
#pragma unroll
      for (int u = 0; u < 16; ++u) v[u] = (f0 + u < p) ? __ldg(src + (int64_t)(f0 + u) * ldx) : 0.0;
#pragma unroll
      for (int u = 0; u < 16; ++u)
        if (f0 + u < p && ok) sx[r * stride + f0 + u] = (f0 + u == mcol) ? vg : v[u];
    }
  }
  __syncthreads();
  double acc = 0.0;
  if ((int)threadIdx.x < rows) {
    const double* x = sx + threadIdx.x * stride;
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
      bool any = true;
      while (any) {
        any = false;
#pragma unroll
        for (int u = 0; u < PILP; ++u)
          if (nd[u].feature >= 0) {
            nd[u] = load_node(tn[u] + (x[nd[u].feature] <= nd[u].v ? nd[u].left : nd[u].left + 1));
            any = true;
          }
      }
#pragma unroll
      for (int u = 0; u < PILP; ++u)
        if (u < na) acc += nd[u].v;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_down_sync(0xffffffffu, acc, o);
  if ((threadIdx.x & 31) == 0) sred[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double tot = 0.0;
    for (int w = 0; w < PT / 32; ++w) tot += sred[w];
    atomicAdd(&pd_sum[blockIdx.y], tot);
  }
}

__global__ void k_pdep_scale(const double* pd_sum, int G, double denom, double* pd) {
  const int g = blockIdx.x * blockDim.x + threadIdx.x;
  if (g < G) pd[g] = __ddiv_rn(pd_sum[g], denom);
}

// R23 grid: G = min(n_pt, distinct values of x); v_g = lo + g * ((hi - lo) / (G - 1)), v_{G-1} = hi.
__global__ void k_sort_key_of(const double* x, int64_t n, uint64_t* keys) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint64_t b = (uint64_t)__double_as_longlong(__dadd_rn(x[i], 0.0));  // -0 -> +0 (R18)
  keys[i] = (b >> 63) ? ~b : (b | 0x8000000000000000ull);               // order-preserving
}
__global__ void k_count_distinct(const uint64_t* keys, int64_t n, unsigned long long* cnt) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const bool d = i < n && (i == 0 || keys[i] != keys[i - 1]);
  const unsigned b = __ballot_sync(0xffffffffu, d);
  if ((threadIdx.x & 31) == 0 && b) atomicAdd(cnt, (unsigned long long)__popc(b));
}
__device__ __forceinline__ double key_to_double(uint64_t k) {
  const uint64_t b = (k >> 63) ? (k & 0x7fffffffffffffffull) : ~k;
  return __longlong_as_double((long long)b);
}
__global__ void k_pd_grid(const uint64_t* sorted, int64_t n, const unsigned long long* cnt, int n_pt, double* grid,
                          int32_t* G_out) {
  const double lo = key_to_double(sorted[0]), hi = key_to_double(sorted[n - 1]);
  const int G = (int)min((unsigned long long)n_pt, *cnt);
  const double by = G > 1 ? __ddiv_rn(__dsub_rn(hi, lo), (double)(G - 1)) : 0.0;
  for (int g = threadIdx.x; g < G; g += blockDim.x)
    grid[g] = (g == G - 1 && G > 1) ? hi : __dadd_rn(lo, __dmul_rn((double)g, by));
  if (threadIdx.x == 0) *G_out = G;
}

}  // namespace

void pd_grid_impl(const double* x_in, int64_t n, int32_t n_pt, double* grid_in, int32_t* G_host, cudaStream_t s) {
  InStage xs(x_in, sizeof(double) * (size_t)n, s);
  OutStage gs(grid_in, sizeof(double) * (size_t)n_pt, s);
  DBuf<uint64_t> keys(n, s), sorted(n, s);
  DBuf<unsigned long long> cnt(1, s);
  DBuf<int32_t> Gd(1, s);
  BF_CUDA_CHECK(cudaMemsetAsync(cnt.p, 0, 8, s));
  {
    KScope ks_("k_sort_key_of", s, 0.0);
    k_sort_key_of<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>((const double*)xs.dptr, n, keys.p);
  }
  const uint64_t* srt = radix_sort_u64(keys.p, sorted.p, nullptr, nullptr, n, 1, s, nullptr);
  {
    KScope ks_("k_count_distinct", s, 0.0);
    k_count_distinct<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>(srt, n, cnt.p);
  }
  {
    KScope ks_("k_pd_grid", s, 0.0);
    k_pd_grid<<<1, 64, 0, s>>>(srt, n, cnt.p, n_pt, (double*)gs.dptr, Gd.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  BF_CUDA_CHECK(cudaMemcpyAsync(G_host, Gd.p, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  gs.finish(s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

void partial_dependence_impl(const bf_forest* f, const double* X_in, int64_t ldx, int64_t n, int32_t mcol,
                             const double* grid_in, int32_t G, double* pd_sum_in, double* pd_in, int32_t ntree_total,
                             cudaStream_t s) {
  const int p = f->info.p;
  const int32_t nt = f->info.tree_end - f->info.tree_begin;
  InStage Xs(X_in, sizeof(double) * (size_t)(ldx * (p - 1) + n), s);
  InStage gs(grid_in, sizeof(double) * (size_t)G, s);
  OutStage ps(pd_sum_in, pd_sum_in ? sizeof(double) * G : 0, s), pp(pd_in, pd_in ? sizeof(double) * G : 0, s);
  DBuf<double> tmp_sum;
  double* psum = pd_sum_in ? (double*)ps.dptr : nullptr;
  if (!psum) {
    tmp_sum.alloc(G, s);
    psum = tmp_sum.p;
  }
  BF_CUDA_CHECK(cudaMemsetAsync(psum, 0, sizeof(double) * G, s));
  const size_t smem = sizeof(double) * (size_t)PT * (size_t)(p | 1);
  static int smax = 0;
  if (!smax) smax = dyn_smem_limit(k_pdep);
  BF_REQUIRE(smem <= (size_t)smax, BF_ENOTIMPL, "bf_partial_dependence: p too large for the shared-memory row tile");
  if (n > 0 && nt > 0) {
    const int64_t block_bytes = 64ll << 20;  // tree blocks L2-resident while every (row tile, g) walks them
    int32_t t0 = 0;
    while (t0 < nt) {
      int32_t t1 = t0 + 1;
      while (t1 < nt && (f->tree_off[t1 + 1] - f->tree_off[t0]) * (int64_t)sizeof(Node16) <= block_bytes) ++t1;
      if (t1 < nt && t1 - t0 > PILP) t1 = t0 + (t1 - t0) / PILP * PILP;
      {
        KScope ks_("k_pdep", s, 0.0);
        k_pdep<<<dim3((unsigned)ceil_div(n, PT), (unsigned)G), PT, smem, s>>>(
            f->d_nodes, f->d_tree_off, t0, t1, (const double*)Xs.dptr, ldx, n, p, mcol, (const double*)gs.dptr, psum);
      }
      t0 = t1;
    }
  }
  if (pd_in) {
    const double denom = (double)n * (double)(ntree_total > 0 ? ntree_total : std::max(nt, 1));
    KScope ks_("k_pdep_scale", s, 0.0);
    k_pdep_scale<<<(unsigned)ceil_div(G, 128), 128, 0, s>>>(psum, G, denom, (double*)pp.dptr);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  if (pd_sum_in) ps.finish(s);
  if (pd_in) pp.finish(s);
  if (ps.host || pp.host || Xs.tmp.p || gs.tmp.p) BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

// Bytes of nodes per tree block (L2-resident while every row walks the block); BF_PREDICT_BLOCK_BYTES
// overrides it (tests force many blocks on small forests).
// Defaults measured on the C4 forest with a 10M-row batch (tools/predict_exp.py): 32 MB of Node8, 48 MB of
// Node16 (larger blocks start to miss in L2, smaller ones re-stage the row tiles too often).
static int64_t predict_block_bytes(int64_t dflt) {
  const char* e = getenv("BF_PREDICT_BLOCK_BYTES");
  const long long v = e ? atoll(e) : 0;
  return v > 0 ? (int64_t)v : dflt;
}

const uint2* nodes8_get(bf_forest* f, cudaStream_t s) {
  if (f->nodes8_state == 0) {
    const int32_t nt = f->info.tree_end - f->info.tree_begin;
    const bool ok = f->info.p <= (1 << N8_FEAT_BITS) && f->info.total_nodes > 0 && nt > 0 &&
                    f->info.total_nodes < (int64_t(1) << 31);
    f->nodes8_state = -1;
    if (ok) {
      f->d_nodes8 = (uint2*)dev_alloc(sizeof(uint2) * (size_t)f->info.total_nodes, s);
      f->d_roots8 = (uint32_t*)dev_alloc(sizeof(uint32_t) * (size_t)nt, s);
      DBuf<int> bad(1, s);
      BF_CUDA_CHECK(cudaMemsetAsync(bad.p, 0, sizeof(int), s));
      {
        KScope ks_("k_pack8", s, 24.0 * (double)f->info.total_nodes);
        k_pack8<<<dim3(64, (unsigned)nt), 256, 0, s>>>(f->d_nodes, f->d_tree_off, f->d_nodes8, f->d_roots8, bad.p);
      }
      BF_CUDA_CHECK(cudaGetLastError());
      int hbad = 0;
      BF_CUDA_CHECK(cudaMemcpyAsync(&hbad, bad.p, sizeof(int), cudaMemcpyDeviceToHost, s));
      BF_CUDA_CHECK(cudaStreamSynchronize(s));
      if (hbad) {
        dev_free(f->d_nodes8, s);
        dev_free(f->d_roots8, s);
        f->d_nodes8 = nullptr;
        f->d_roots8 = nullptr;
      } else {
        f->nodes8_state = 1;
      }
    }
  }
  return f->nodes8_state > 0 ? f->d_nodes8 : nullptr;
}


const ulonglong4* g32_get(bf_forest* f, cudaStream_t s) {
  if (f->g32_state == 0) {
    const int32_t nt = f->info.tree_end - f->info.tree_begin;
    const int64_t total = f->info.total_nodes;
    f->g32_state = -1;
    if (f->info.p <= 256 && total > 0 && nt > 0 && total < (int64_t(1) << 31)) {
      DBuf<int32_t> anc0(total, s), anc1(total, s);
      DBuf<uint8_t> bit0(total, s), bit1(total, s);
      DBuf<int> flag(2, s);
      const dim3 tg(64, (unsigned)nt);
      {
        KScope ks_("k_g32_build", s, 0.0);
        k_g32_parent<<<tg, 256, 0, s>>>(f->d_nodes, f->d_tree_off, anc0.p, bit0.p);
      }
      BF_CUDA_CHECK(cudaGetLastError());
      int32_t* a = anc0.p;
      int32_t* a2 = anc1.p;
      uint8_t* b = bit0.p;
      uint8_t* b2 = bit1.p;
      for (int it = 0; it < 40; ++it) {  // depth < 2^40: ends when every node's ancestor link is the root's
        int more = 0;
        BF_CUDA_CHECK(cudaMemsetAsync(flag.p, 0, sizeof(int), s));
        {
          KScope ks_("k_g32_build", s, 0.0);
          k_g32_jump<<<(unsigned)ceil_div(total, 256), 256, 0, s>>>(a, b, a2, b2, total, flag.p);
        }
        BF_CUDA_CHECK(cudaMemcpyAsync(&more, flag.p, sizeof(int), cudaMemcpyDeviceToHost, s));
        BF_CUDA_CHECK(cudaStreamSynchronize(s));
        std::swap(a, a2);
        std::swap(b, b2);
        if (!more) break;
      }
      uint32_t* cnt = reinterpret_cast<uint32_t*>(a2);  // the other ancestor buffer is free now
      uint32_t* ex = reinterpret_cast<uint32_t*>(a);
      DBuf<int64_t> tslot((size_t)nt + 1, s);
      {
        KScope ks_("k_g32_build", s, 0.0);
        k_g32_count<<<tg, 256, 0, s>>>(f->d_nodes, f->d_tree_off, b, cnt);
      }
      DBuf<uint32_t> exb(total, s);
      scan_exclusive(cnt, exb.p, total, s);
      uint32_t last_ex = 0, last_cnt = 0;
      BF_CUDA_CHECK(cudaMemcpyAsync(&last_ex, exb.p + total - 1, 4, cudaMemcpyDeviceToHost, s));
      BF_CUDA_CHECK(cudaMemcpyAsync(&last_cnt, cnt + total - 1, 4, cudaMemcpyDeviceToHost, s));
      BF_CUDA_CHECK(cudaStreamSynchronize(s));
      const int64_t nslots = (int64_t)last_ex + last_cnt;
      {
        KScope ks_("k_g32_build", s, 0.0);
        k_g32_slots<<<tg, 256, 0, s>>>(f->d_nodes, f->d_tree_off, b, exb.p, ex, tslot.p);
      }
      f->d_g32 = (ulonglong4*)dev_alloc(sizeof(ulonglong4) * (size_t)nslots, s);
      f->d_g32_root = (uint32_t*)dev_alloc(sizeof(uint32_t) * (size_t)nt, s);
      BF_CUDA_CHECK(cudaMemsetAsync(flag.p + 1, 0, sizeof(int), s));
      {
        KScope ks_("k_g32_build", s, 0.0);
        k_g32_emit<<<tg, 256, 0, s>>>(f->d_nodes, f->d_tree_off, b, exb.p, ex, f->d_g32, f->d_g32_root, flag.p + 1);
      }
      BF_CUDA_CHECK(cudaGetLastError());
      f->g32_off.assign((size_t)nt + 1, 0);
      int hbad = 0;
      BF_CUDA_CHECK(cudaMemcpyAsync(f->g32_off.data(), tslot.p, sizeof(int64_t) * nt, cudaMemcpyDeviceToHost, s));
      BF_CUDA_CHECK(cudaMemcpyAsync(&hbad, flag.p + 1, sizeof(int), cudaMemcpyDeviceToHost, s));
      BF_CUDA_CHECK(cudaStreamSynchronize(s));
      f->g32_off[nt] = nslots;
      if (hbad || nslots >= (int64_t(1) << 31)) {
        dev_free(f->d_g32, s);
        dev_free(f->d_g32_root, s);
        f->d_g32 = nullptr;
        f->d_g32_root = nullptr;
      } else {
        f->g32_state = 1;
      }
    }
  }
  return f->g32_state > 0 ? f->d_g32 : nullptr;
}

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
    vis.alloc(2, s);
    BF_CUDA_CHECK(cudaMemsetAsync(vis.p, 0, 16, s));
  }
  const char* force16 = getenv("BF_PREDICT_NODE16");
  const uint2* n8 = (force16 && force16[0] == '1') ? nullptr : nodes8_get(const_cast<bf_forest*>(f), s);
  const size_t smem8 = sizeof(float) * (size_t)PT8 * (size_t)(p | 1);
  static int smax8 = 0;
  if (!smax8) {
    smax8 = std::min(dyn_smem_limit(k_predict8<true>), dyn_smem_limit(k_predict8<false>));
    smax8 = std::min(smax8, std::min(dyn_smem_limit(k_predict8s<true, 6>), dyn_smem_limit(k_predict8s<false, 6>)));
    smax8 = std::min(smax8, std::min(dyn_smem_limit(k_predict8s<true, 8>), dyn_smem_limit(k_predict8s<false, 8>)));
    smax8 = std::min(smax8, std::min(dyn_smem_limit(k_predict8s<true, 12>), dyn_smem_limit(k_predict8s<false, 12>)));
  }
  static const int slots = getenv("BF_PREDICT_SLOTS") ? atoi(getenv("BF_PREDICT_SLOTS")) : 6;  // measured: 6 < 8 < 12 (profiles/r02o)
  // walk kernel: 3 = G32 groups, 2 = Node8 with the block's roots in shared memory, 1 = Node8 (read per call,
  // so tests can compare the paths on one forest)
  const int pv = getenv("BF_PREDICT_V") ? atoi(getenv("BF_PREDICT_V")) : 3;
  static int smax32 = 0;
  if (!smax32)
    smax32 = std::min(std::min(std::min(dyn_smem_limit(k_predict32<true, 4>), dyn_smem_limit(k_predict32<false, 4>)),
                               std::min(dyn_smem_limit(k_predict32<true, 6>), dyn_smem_limit(k_predict32<false, 6>))),
                      std::min(dyn_smem_limit(k_predict32<true, 5>), dyn_smem_limit(k_predict32<false, 5>)));
  const ulonglong4* g32 = (pv == 3 && !(force16 && force16[0] == '1')) ? g32_get(const_cast<bf_forest*>(f), s) : nullptr;
  if (g32 && smem8 <= (size_t)smax32) {
    // G32 groups: tree blocks of <= 48 MB of slots (one 256-bit load per two levels)
    double* ysum = ys_in ? (double*)ys.dptr : nullptr;
    DBuf<double> ytmp;
    if (!ysum) {
      ytmp.alloc(m, s);
      ysum = ytmp.p;
    }
    static const int slots32 = getenv("BF_PREDICT32_SLOTS") ? atoi(getenv("BF_PREDICT32_SLOTS")) : 4;
    const int64_t block_bytes = predict_block_bytes(48ll << 20);
    // with more than one tree block the row tiles are staged once per block: from a row-major float copy of
    // the query batch (half the bytes of the fp64 columns, contiguous per row), built once per call
    static const int use_xf = getenv("BF_PREDICT_XF") ? atoi(getenv("BF_PREDICT_XF")) : 0;  // measured: no gain (189 vs 188 ms per 200 C4 trees)
    const int xfs = (p + 3) & ~3;
    DBuf<float> Xqf;
    if (use_xf && f->g32_off[nt] * (int64_t)sizeof(ulonglong4) > block_bytes) {
      Xqf.alloc((size_t)m * xfs, s);
      xf_rows_impl((const double*)Xs.dptr, ldq, m, p, Xqf.p, xfs, s);
    }
    for (int32_t t0 = 0; t0 < nt;) {
      int32_t t1 = t0 + 1;
      while (t1 < nt && t1 - t0 < RT8 && (f->g32_off[t1 + 1] - f->g32_off[t0]) * (int64_t)sizeof(ulonglong4) <= block_bytes) ++t1;
      KScope ks_("k_predict32", s, 0.0);
      auto kern = vis.p ? (slots32 == 6 ? k_predict32<true, 6> : slots32 == 5 ? k_predict32<true, 5> : k_predict32<true, 4>)
                        : (slots32 == 6 ? k_predict32<false, 6> : slots32 == 5 ? k_predict32<false, 5> : k_predict32<false, 4>);
      kern<<<(unsigned)ceil_div(m, PT8), PT8, smem8, s>>>(g32, f->d_nodes, f->d_g32_root, t0, t1, t0 == 0, t1 >= nt,
                                                         (const double*)Xs.dptr, ldq, Xqf.p, xfs, m, p, ysum,
                                                         yh_in ? (double*)yh.dptr : nullptr, inv_t, vis.p);
      t0 = t1;
    }
  } else if (n8 && smem8 <= (size_t)smax8) {
    // tree blocks of <= 32 MB of Node8 (L2-resident while every row walks them)
    double* ysum = ys_in ? (double*)ys.dptr : nullptr;
    DBuf<double> ytmp;
    if (!ysum) {
      ytmp.alloc(m, s);
      ysum = ytmp.p;
    }
    const int64_t block_bytes = predict_block_bytes(32ll << 20);
    for (int32_t t0 = 0; t0 < nt;) {
      int32_t t1 = t0 + 1;
      while (t1 < nt && (f->tree_off[t1 + 1] - f->tree_off[t0]) * (int64_t)sizeof(uint2) <= block_bytes) ++t1;
      if (t1 - t0 <= RT8 && pv != 1) {
        KScope ks_("k_predict8", s, 0.0);
        auto kern = vis.p ? (slots == 6 ? k_predict8s<true, 6> : slots == 12 ? k_predict8s<true, 12> : k_predict8s<true, 8>)
                          : (slots == 6 ? k_predict8s<false, 6> : slots == 12 ? k_predict8s<false, 12> : k_predict8s<false, 8>);
        kern<<<(unsigned)ceil_div(m, PT8), PT8, smem8, s>>>(
            n8, f->d_nodes, f->d_roots8, t0, t1, t0 == 0, t1 >= nt, (const double*)Xs.dptr, ldq, m, p, ysum,
            yh_in ? (double*)yh.dptr : nullptr, inv_t, vis.p);
      } else {
        KScope ks_("k_predict8", s, 0.0);
        (vis.p ? k_predict8<true> : k_predict8<false>)<<<(unsigned)ceil_div(m, PT8), PT8, smem8, s>>>(
            n8, f->d_nodes, f->d_roots8, t0, t1, t0 == 0, t1 >= nt, (const double*)Xs.dptr, ldq, m, p, ysum,
            yh_in ? (double*)yh.dptr : nullptr, inv_t, vis.p);
      }
      t0 = t1;
    }
  } else if (smem <= (size_t)smax) {
    // tree blocks of <= 64 MB of nodes (L2-resident while every row walks them)
    double* ysum = ys_in ? (double*)ys.dptr : nullptr;
    DBuf<double> ytmp;
    if (!ysum) {
      ytmp.alloc(m, s);
      ysum = ytmp.p;
    }
    const int64_t block_bytes = predict_block_bytes(48ll << 20);
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
    unsigned long long hv2[2] = {0, 0};
    BF_CUDA_CHECK(cudaMemcpyAsync(hv2, vis.p, 16, cudaMemcpyDeviceToHost, s));
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
    const unsigned long long hv = hv2[0];
    prof_add_bytes("predict_node_visits", (double)hv);
    prof_add_bytes("predict_fp64_fallbacks", (double)hv2[1]);
    const bool used32 = g32 && smem8 <= (size_t)smax32;
    const bool used8 = !used32 && n8 && smem8 <= (size_t)smax8;
    prof_add_bytes(used32 ? "k_predict32" : used8 ? "k_predict8" : smem <= (size_t)smax ? "k_predict_smem" : "k_predict_gmem",
                   (used32 ? 32.0 : used8 ? 8.0 : 16.0) * (double)hv +
                       (double)m * (8.0 * p + 16.0 * ((ys_in != nullptr) + (yh_in != nullptr))));
  }
  if (ys_in) ys.finish(s);
  if (yh_in) yh.finish(s);
  if (ys.host || yh.host || Xs.tmp.p) BF_CUDA_CHECK(cudaStreamSynchronize(s));
}

}  // namespace bf
