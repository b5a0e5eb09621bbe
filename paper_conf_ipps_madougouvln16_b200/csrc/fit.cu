// fit.cu -- forest construction on sm_100a.
//
// Design:
//   once per fit   a1 validate, a2 fixed-point y_q, a3 presort: per feature the
//                  rows in x order (CUB radix sort of order-preserving keys),
//                  the dense rank of every value and the table of distinct values.
//   per batch of B trees in flight:
//     a4 bootstrap multiplicities (Philox BOOT), root sums;
//     a5 root lists: per (tree, feature) stable compaction of the presorted
//        column to the in-bag rows, 8-byte entries rank|row|w (node-major
//        block: p segments of a entries, each in value order);
//     GLOBAL PHASE (nodes with more than A distinct rows), level-synchronous
//     over all trees of the batch:
//        a6 k_mtry; a7 k_split_scan_tree (tree-affine CTAs own whole
//        (node, drawn feature) items: TMA-staged units, segmented prefix scan
//        of (w, w*y_q) with a carry, rigorous fp64 screen, exact key near the
//        max); a8 k_finalize + CUB scans + k_child_place; a9/a10 k_dest_bits
//        (goes-right bitmap of the winning segments + child sums of w*y) and
//        k_child_values; a9 k_partition_tree (tree-affine CTAs, goes-right
//        bitmap in shared memory, stable partition of all p segments into the
//        children's blocks, small children to the subtree queue);
//     SUBTREE PHASE (nodes with <= A distinct rows): one CTA grows the whole
//        subtree in shared memory (k_subtree: medium levels with in-place
//        nested ranges, then tiny nodes of <= 64 rows as bit masks over their
//        tiny root's sorted segments, through a CTA work queue);
//     a11 k_emit: raw per-tree pools -> packed node arrays (root 0, right =
//        left + 1; slot order is allocation order, not BFS: DESIGN.md R21).
// All split arithmetic is exact (int64 sums, int128 D, correctly rounded
// key) so the topology is bit-identical to the CPU oracle whatever the scan
// order, tile size or number of GPUs.
#include <cuda/atomic>

#include <mutex>

#include <algorithm>
#include <cstdio>
#include <ctime>
#include <cstdlib>
#include <cmath>
#include <cstring>

#include "bf_internal.cuh"

namespace bf {

namespace {

constexpr int NT = 256;         // threads per CTA of the streaming kernels
constexpr int SUB_NW = 16;      // warps of the subtree kernel
constexpr int SUB_NT = SUB_NW * 32;
constexpr int KIND_NONE = -1, KIND_LEAF = 0, KIND_SMALL = 1, KIND_LARGE = 2;

// List entry (8 B): dense rank of the value (24 bits) | row (24 bits) | bootstrap
// multiplicity w (16 bits).  Entries of a segment are kept in value order, so the
// scan reads w from the entry and gathers only y_q[row] (one 8 MB array shared
// by every tree: L2-resident) instead of a per-tree payload.
__host__ __device__ __forceinline__ uint32_t e_rank(uint64_t e) { return (uint32_t)(e >> 40); }
__host__ __device__ __forceinline__ uint32_t e_row(uint64_t e) { return (uint32_t)(e >> 16) & 0xffffffu; }
__host__ __device__ __forceinline__ int32_t e_w(uint64_t e) { return (int32_t)(e & 0xffffu); }
constexpr int64_t MAX_ROWS = int64_t(1) << 24;

struct LNode {  // an active node of the global phase, or a queued small node
  int32_t b;     // tree index inside the batch
  int32_t raw;   // node slot in the tree's raw pool
  int32_t a;     // distinct in-bag rows
  int32_t n;     // n_k = sum of w
  int64_t S;     // S_k = sum of w * y_q
  uint64_t key;  // node path key (S3 KEY)
  int64_t base;  // element offset of the node's block (p segments of a entries)
};

struct Rec {  // best candidate of one (node, drawn feature)
  double g;
  uint32_t rank_a, rank_b;  // dense ranks of the values left / right of the boundary
  int32_t pos;              // boundary position (last left entry) inside the segment
  int32_t nl;
  int64_t Sl;
};

struct Split {
  int32_t split;  // 0 leaf, 1 split
  int32_t f, pos, lraw;
  int32_t nl, nr;
  int32_t pad0, pad1;
};

struct Child {
  int32_t kind, a, n, raw;
  int64_t S;
  uint64_t key;
  int64_t base;
};

struct Pool {  // raw per-tree node pool of a batch (capacity `cap` per tree)
  int32_t* feature;
  int32_t* left;
  int32_t* count;
  double* thr;
  double* value;
  double* drss;
  int32_t* nn;   // nodes used per tree
  int64_t cap;
};

struct LevelSummary {
  int32_t nnext;      // large nodes of the next level
  int32_t nsmall;     // queued small nodes (total)
  int64_t small_elems;  // elements used in the small-node area (total)
  int64_t next_elems;   // elements of the next level's blocks
  unsigned long long split_a;  // sum of a over the nodes split at this level
  unsigned long long pad;
};

// ------------------------------------------------------------------ warp / block scans
template <class T>
__device__ __forceinline__ T warp_incl_scan(T v, int lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T u = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += u;
  }
  return v;
}

// Exclusive block scan; `sm` holds NT/32 elements; returns exclusive prefix and total.
template <class T>
__device__ __forceinline__ T block_excl_scan(T v, T* sm, T& total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  T inc = warp_incl_scan(v, lane);
  if (lane == 31) sm[wid] = inc;
  __syncthreads();
  if (wid == 0) {
    T s = lane < nw ? sm[lane] : T(0);
    s = warp_incl_scan(s, lane);
    if (lane < nw) sm[lane] = s;
  }
  __syncthreads();
  T pre = wid ? sm[wid - 1] : T(0);
  total = sm[nw - 1];
  __syncthreads();
  return pre + inc - v;
}

// ------------------------------------------------------------------ a1 validate
__global__ void k_validate(const double* X, int64_t ldx, int64_t n, int32_t p, const double* y, int* bad) {
  const int64_t total = n * (int64_t)p;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total + n; i += (int64_t)gridDim.x * blockDim.x) {
    double v;
    if (i < total) {
      const int64_t j = i / n, r = i - j * n;
      v = X[j * ldx + r];
    } else {
      v = y[i - total];
    }
    if (!isfinite(v)) atomicOr(bad, 1);
  }
}

// ------------------------------------------------------------------ a2 fixed point
__global__ void k_minmax(const double* y, int64_t n, double* part) {  // part[2*blk] = min, max
  __shared__ double smin[NT], smax[NT];
  double mn = INFINITY, mx = -INFINITY;
  for (int64_t i = blockIdx.x * (int64_t)NT + threadIdx.x; i < n; i += (int64_t)gridDim.x * NT) {
    mn = fmin(mn, y[i]);
    mx = fmax(mx, y[i]);
  }
  smin[threadIdx.x] = mn;
  smax[threadIdx.x] = mx;
  __syncthreads();
  for (int s = NT / 2; s > 0; s >>= 1) {
    if (threadIdx.x < s) {
      smin[threadIdx.x] = fmin(smin[threadIdx.x], smin[threadIdx.x + s]);
      smax[threadIdx.x] = fmax(smax[threadIdx.x], smax[threadIdx.x + s]);
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    part[2 * blockIdx.x] = smin[0];
    part[2 * blockIdx.x + 1] = smax[0];
  }
}

__global__ void k_absdev_max(const double* y, int64_t n, double c, double* part) {
  __shared__ double sm[NT];
  double mx = 0.0;
  for (int64_t i = blockIdx.x * (int64_t)NT + threadIdx.x; i < n; i += (int64_t)gridDim.x * NT)
    mx = fmax(mx, fabs(__dsub_rn(y[i], c)));
  sm[threadIdx.x] = mx;
  __syncthreads();
  for (int s = NT / 2; s > 0; s >>= 1) {
    if (threadIdx.x < s) sm[threadIdx.x] = fmax(sm[threadIdx.x], sm[threadIdx.x + s]);
    __syncthreads();
  }
  if (threadIdx.x == 0) part[blockIdx.x] = sm[0];
}

__global__ void k_yq(const double* y, int64_t n, double c, int q, int zero, int64_t* yq) {
  for (int64_t i = blockIdx.x * (int64_t)NT + threadIdx.x; i < n; i += (int64_t)gridDim.x * NT)
    yq[i] = zero ? 0 : __double2ll_rn(ldexp(__dsub_rn(y[i], c), q));
}

// ------------------------------------------------------------------ a3 presort
// All p features at once (feature-major arrays of p * n): order-preserving 64-bit keys of the canonical
// values (-0 -> +0), one segmented radix sort (prims.cu), dense ranks by a scan of the value-change flags.
__global__ void k_sort_keys(const double* X, int64_t ldx, int64_t n, int p, uint64_t* keys, uint32_t* vals) {
  const int64_t tot = n * p;
  for (int64_t k = blockIdx.x * (int64_t)NT + threadIdx.x; k < tot; k += (int64_t)gridDim.x * NT) {
    const int64_t f = k / n, i = k - f * n;
    const uint64_t b = (uint64_t)__double_as_longlong(canon(X[f * ldx + i]));
    keys[k] = (b >> 63) ? ~b : (b | 0x8000000000000000ull);  // order-preserving
    vals[k] = (uint32_t)i;
  }
}

__global__ void k_rank_flags(const uint64_t* keys, int64_t n, int p, uint32_t* flags) {
  const int64_t tot = n * p;
  for (int64_t k = blockIdx.x * (int64_t)NT + threadIdx.x; k < tot; k += (int64_t)gridDim.x * NT) {
    const int64_t i = k % n;
    flags[k] = (i > 0 && keys[k] != keys[k - 1]) ? 1u : 0u;
  }
}

// rank: inclusive scan of the flags over all features; feature f's dense ranks are rank - rank[f * n].
__global__ void k_fill_sorted(const double* X, int64_t ldx, const uint32_t* rows, const uint32_t* rank, int64_t n,
                              int p, uint64_t* srt, double* uniq) {
  const int64_t tot = n * p;
  for (int64_t k = blockIdx.x * (int64_t)NT + threadIdx.x; k < tot; k += (int64_t)gridDim.x * NT) {
    const int64_t f = k / n, i = k - f * n;
    const uint32_t r = rows[k], rk = rank[k] - rank[f * n];
    srt[k] = ((uint64_t)rk << 40) | ((uint64_t)r << 16);
    if (i == 0 || rank[k - 1] != rank[k]) uniq[f * n + rk] = canon(X[f * ldx + r]);
  }
}

// ------------------------------------------------------------------ a4 bootstrap
__global__ void k_bootstrap(uint64_t seed, int32_t t0, int64_t n, int64_t ns, int32_t* w) {
  const int b = blockIdx.y;
  const uint32_t t = (uint32_t)(t0 + b);
  const int64_t j2 = blockIdx.x * (int64_t)NT + threadIdx.x;
  if (2 * j2 >= ns) return;
  uint64_t u0, u1;
  philox_u64x2(seed, (uint32_t)j2, t, 1u, 0u, u0, u1);
  int32_t* wb = w + (int64_t)b * n;
  atomicAdd(&wb[mulhi64(u0, (uint64_t)n)], 1);
  if (2 * j2 + 1 < ns) atomicAdd(&wb[mulhi64(u1, (uint64_t)n)], 1);
}

__global__ void k_fill_i32(int32_t* a, int64_t count, int32_t v) {
  for (int64_t i = blockIdx.x * (int64_t)NT + threadIdx.x; i < count; i += (int64_t)gridDim.x * NT) a[i] = v;
}

// payload + per-tree root sums: a (distinct), S (exact), sum w*y (fp64)
__global__ void k_payload(const int32_t* w, const int64_t* yq, const double* y, int64_t n, int32_t* wmax,
                          int32_t* a_root, unsigned long long* S_root, double* sy_root) {
  __shared__ int32_t sa[NT / 32];
  __shared__ int64_t sS[NT / 32];
  __shared__ double sy[NT / 32];
  const int b = blockIdx.y;
  const int64_t i = blockIdx.x * (int64_t)NT + threadIdx.x;
  int32_t wi = 0;
  int64_t wyq = 0;
  double wy = 0.0;
  if (i < n) {
    wi = w[(int64_t)b * n + i];
    wyq = (int64_t)wi * yq[i];
    wy = __dmul_rn((double)wi, y[i]);
    if (wi > 0xffff) atomicMax(wmax, wi);
  }
  int32_t ca = wi > 0;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    ca += __shfl_down_sync(0xffffffffu, ca, o);
    wyq += __shfl_down_sync(0xffffffffu, wyq, o);
    wy += __shfl_down_sync(0xffffffffu, wy, o);
  }
  if (lane == 0) {
    sa[wid] = ca;
    sS[wid] = wyq;
    sy[wid] = wy;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int32_t A = 0;
    int64_t S = 0;
    double Y = 0.0;
    for (int k = 0; k < NT / 32; ++k) {
      A += sa[k];
      S += sS[k];
      Y += sy[k];
    }
    atomicAdd(&a_root[b], A);
    atomicAdd(&S_root[b], (unsigned long long)S);
    atomicAdd(&sy_root[b], Y);
  }
}

// root records + root node descriptors
__global__ void k_roots(int B, int64_t ns, int nodesize, const int32_t* a_root, const unsigned long long* S_root,
                        const double* sy_root, const int32_t* kind, const int64_t* base, Pool pool, LNode* lroots,
                        int32_t* lidx, LNode* sq, int32_t* sidx) {
  const int b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= B) return;
  const int64_t r0 = (int64_t)b * pool.cap;
  pool.feature[r0] = -1;
  pool.left[r0] = -1;
  pool.count[r0] = (int32_t)ns;
  pool.thr[r0] = 0.0;
  pool.value[r0] = __ddiv_rn(sy_root[b], (double)ns);
  pool.drss[r0] = 0.0;
  pool.nn[b] = 1;
  LNode nd;
  nd.b = b;
  nd.raw = 0;
  nd.a = a_root[b];
  nd.n = (int32_t)ns;
  nd.S = (int64_t)S_root[b];
  nd.key = 0;
  nd.base = base[b];
  if (kind[b] == KIND_LARGE) lroots[lidx[b]] = nd;
  if (kind[b] == KIND_SMALL) sq[sidx[b]] = nd;
}

// ------------------------------------------------------------------ a5 root lists (two-pass stable compaction)
constexpr int LCH = 2048;  // entries per CTA chunk (256 threads x 8)

// The batch's multiplicities row-major as uint16 (w <= 65535 is checked after k_payload): wp[row * Bp + b],
// Bp = B rounded up to LTG, so one 32-byte load gives a row's weights for LTG trees (16 trees per pass over the
// presorted columns: 3 passes for a 37-tree batch instead of 5 with 16-byte loads of 8 trees).
constexpr int LTG = 16;  // trees per list-init CTA
__global__ void k_w_pack(const int32_t* w, int64_t n, int B, int Bp, uint16_t* wp) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint16_t v[8];
  for (int b0 = 0; b0 < Bp; b0 += 8) {
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = b0 + u < B ? (uint16_t)w[(int64_t)(b0 + u) * n + i] : (uint16_t)0;
    uint4 q;
    q.x = v[0] | ((uint32_t)v[1] << 16);
    q.y = v[2] | ((uint32_t)v[3] << 16);
    q.z = v[4] | ((uint32_t)v[5] << 16);
    q.w = v[6] | ((uint32_t)v[7] << 16);
    *reinterpret_cast<uint4*>(wp + i * Bp + b0) = q;
  }
}
using WQ = ulonglong4;  // a row's weights for LTG trees
__device__ __forceinline__ WQ wp_load(const uint16_t* p) { return ldg256(reinterpret_cast<const ulonglong4*>(p)); }
__device__ __forceinline__ uint32_t wp_get(const WQ& q, int u) {
  const unsigned long long w4 = u < 4 ? q.x : u < 8 ? q.y : u < 12 ? q.z : q.w;
  return (uint32_t)(w4 >> (16 * (u & 3))) & 0xffffu;
}

// One CTA = one chunk of one presorted column for LTG trees of the batch (blockIdx.z = tree group): the
// chunk is read once per group and each entry's weights for the group are ONE 16-byte gather.
__global__ void k_list_count(const uint64_t* srt, int64_t n, const uint16_t* wp, int Bp, const int32_t* kind,
                             int nchunk, int B, int32_t* cnt) {
  const int c = blockIdx.x, f = blockIdx.y, b0 = blockIdx.z * LTG, p = gridDim.y;
  __shared__ int32_t sm[NT / 32];
  constexpr int V = LCH / NT;
  const uint64_t* col = srt + (int64_t)f * n;
  const int64_t i0 = (int64_t)c * LCH + (int64_t)threadIdx.x * V;
  WQ q[V];
#pragma unroll
  for (int u = 0; u < V; ++u)
    q[u] = i0 + u < n ? wp_load(wp + (int64_t)e_row(col[i0 + u]) * Bp + b0) : make_ulonglong4(0ull, 0ull, 0ull, 0ull);
  for (int t = 0; t < LTG && b0 + t < B; ++t) {
    const int b = b0 + t;
    if (kind[b] != KIND_LARGE && kind[b] != KIND_SMALL) continue;  // uniform per CTA
    int32_t k = 0;
#pragma unroll
    for (int u = 0; u < V; ++u) k += wp_get(q[u], t) > 0;
    int32_t tot;
    block_excl_scan(k, sm, tot);
    if (threadIdx.x == 0) cnt[((int64_t)b * p + f) * nchunk + c] = tot;
  }
}

__global__ void k_list_prefix(int32_t* cnt, int nseg, int nchunk) {
  const int s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= nseg) return;
  int32_t* c = cnt + (int64_t)s * nchunk;
  int32_t acc = 0;
  for (int i = 0; i < nchunk; ++i) {
    int32_t v = c[i];
    c[i] = acc;
    acc += v;
  }
}

// Warp w of the CTA owns the chunk's entries [w * 256, (w + 1) * 256), read in rounds of 32 (entry
// w * 256 + 32 u + lane): per round the in-bag entries of one tree are consecutive in the output, so every store
// instruction writes one contiguous run; one block barrier per tree for the warps' in-bag counts.
__global__ void k_list_scatter(const uint64_t* srt, int64_t n, const uint16_t* wp, int Bp, const int32_t* kind,
                               const int64_t* base, const int32_t* a_root, int nchunk, int B, const int32_t* cnt,
                               uint64_t* Elarge, uint64_t* Esmall) {
  const int c = blockIdx.x, f = blockIdx.y, b0 = blockIdx.z * LTG, p = gridDim.y;
  constexpr int V = LCH / NT, NW = NT / 32;
  __shared__ int32_t sm[2][NW];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const uint64_t* col = srt + (int64_t)f * n;
  const int64_t i0 = (int64_t)c * LCH + (int64_t)wid * (V * 32) + lane;
  uint64_t e[V];
  WQ q[V];
#pragma unroll
  for (int u = 0; u < V; ++u) e[u] = i0 + 32 * u < n ? col[i0 + 32 * u] : ~0ull;
#pragma unroll
  for (int u = 0; u < V; ++u)
    q[u] = e[u] != ~0ull ? wp_load(wp + (int64_t)e_row(e[u]) * Bp + b0) : make_ulonglong4(0ull, 0ull, 0ull, 0ull);
  const uint32_t ltm = (1u << lane) - 1u;
  int par = 0;
  for (int t = 0; t < LTG && b0 + t < B; ++t) {
    const int b = b0 + t;
    const int kd = kind[b];
    if (kd != KIND_LARGE && kd != KIND_SMALL) continue;  // uniform per CTA
    uint32_t m[V];
    int32_t wc = 0;
#pragma unroll
    for (int u = 0; u < V; ++u) {
      m[u] = __ballot_sync(0xffffffffu, wp_get(q[u], t) > 0);
      wc += __popc(m[u]);
    }
    if (lane == 0) sm[par][wid] = wc;
    __syncthreads();  // sm[par] is next written two trees later, after another barrier
    int32_t pre = cnt[((int64_t)b * p + f) * nchunk + c];
#pragma unroll
    for (int k = 0; k < NW; ++k)
      if (k < wid) pre += sm[par][k];
    par ^= 1;
    uint64_t* dst = (kd == KIND_LARGE ? Elarge : Esmall) + base[b] + (int64_t)f * a_root[b] + pre;
    int run = 0;
#pragma unroll
    for (int u = 0; u < V; ++u) {
      if ((m[u] >> lane) & 1u) dst[run + __popc(m[u] & ltm)] = e[u] | (uint64_t)wp_get(q[u], t);
      run += __popc(m[u]);
    }
  }
}

__global__ void k_mtry(const LNode* nodes, int N, int p, int mtry, uint64_t seed, int32_t t0, int32_t* feat,
                       int16_t* scratch) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= N) return;
  const LNode nd = nodes[k];
  int16_t* mind = scratch + (int64_t)k * p;
  for (int j = 0; j < p; ++j) mind[j] = (int16_t)j;
  int last = p - 1;
  uint64_t u0 = 0, u1 = 0;
  for (int i = 0; i < mtry; ++i) {
    if ((i & 1) == 0)
      philox_u64x2(seed, (uint32_t)nd.key, (uint32_t)(nd.key >> 32), (uint32_t)(t0 + nd.b),
                   0x20000000u | (uint32_t)(i >> 1), u0, u1);
    const uint64_t u = (i & 1) ? u1 : u0;
    const int j = (int)mulhi64(u, (uint64_t)(last + 1));
    feat[(int64_t)k * mtry + i] = mind[j];
    const int16_t tmp = mind[j];
    mind[j] = mind[last];
    mind[last] = tmp;
    --last;
  }
}

// ------------------------------------------------------------------ a7 split scan (global phase)
// One CTA per (node, drawn feature): chunked segmented scan with a carry.
constexpr int SV = 4;            // entries per thread per chunk
constexpr int SCH = NT * SV;     // 1024 entries per chunk

__device__ __forceinline__ bool rec_better(double g, uint32_t r, double bg, uint32_t br) {
  return g > bg || (g == bg && r < br);
}

// Screen of a candidate against the running best key, in fp64 with a
// rigorous bound (no int128): d = RN(RN(nk*Sl) - RN(nl*Sk)) satisfies
// |d - D| <= 2^-50 (|nk*Sl| + |nl*Sk|), so gU = (|d| + E)^2 * rcp(nn) * (1 + 2^-20)
// bounds the exact D^2/(nl*nr) from above.  Returns false only if the
// correctly rounded key of S4.3 is certainly below `best`.
__device__ __forceinline__ bool screen_may_win(int64_t nk, int64_t Sk, int64_t nl, int64_t Sl, double best) {
  if (best <= 0.0) return true;
  const double a = (double)nk * (double)Sl, bb = (double)nl * (double)Sk;
  const double d = fabs(a - bb);
  const double E = (fabs(a) + fabs(bb)) * 8.881784197001252e-16;  // 2^-50
  const double u = (d + E) * (1.0 + 8.881784197001252e-16);
  const double nn = (double)(nl * (nk - nl));
  const double gU = u * u * (double)__frcp_rn((float)nn) * (1.0 + 9.5367431640625e-07);  // (1 + 2^-20)
  return gU >= best;
}

// Warp argmax of (key desc, tie asc) with 64-bit keys (0 = no candidate):
// returns the winning lane (or -1).  key = bits(g) + 1 for a candidate with
// key g >= 0, which preserves the order of non-negative doubles.
__device__ __forceinline__ int warp_argmax_key(uint64_t key, uint32_t tie) {
  const uint32_t hi = (uint32_t)(key >> 32), lo = (uint32_t)key;
  const uint32_t mh = __reduce_max_sync(0xffffffffu, hi);
  const uint32_t ml = __reduce_max_sync(0xffffffffu, hi == mh ? lo : 0u);
  if (mh == 0 && ml == 0) return -1;
  const bool top = hi == mh && lo == ml;
  const uint32_t mt = __reduce_min_sync(0xffffffffu, top ? tie : 0xffffffffu);
  return __ffs(__ballot_sync(0xffffffffu, top && tie == mt)) - 1;
}
__device__ __forceinline__ uint64_t gkey(double g) { return g >= 0.0 ? (uint64_t)__double_as_longlong(g) + 1ull : 0ull; }


// ------------------------------------------------------------------ a8 node finalize (global phase)
__global__ void k_finalize(const LNode* nodes, int N, const int32_t* feat, const Rec* rec, int mtry,
                           const double* uniq, int64_t n, int nodesize, int Asmall, int q, uint64_t seed,
                           int32_t t0, Pool pool, Split* split, Child* child, uint64_t* packL, uint64_t* packS,
                           LevelSummary* sum) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= N) return;
  const LNode nd = nodes[k];
  double bg = -1.0;
  int bf = 0x7fffffff;
  Rec br;
  br.g = -1.0;
  for (int s = 0; s < mtry; ++s) {
    const Rec R = rec[(int64_t)k * mtry + s];
    const int f = feat[(int64_t)k * mtry + s];
    if (R.g < 0) continue;
    if (R.g > bg || (R.g == bg && f < bf)) {
      bg = R.g;
      bf = f;
      br = R;
    }
  }
  Split sp;
  sp.split = 0;
  sp.pad0 = sp.pad1 = 0;
  Child cl, cr;
  cl.kind = cr.kind = KIND_NONE;
  if (bg > 0.0) {
    const double xa = uniq[(int64_t)bf * n + br.rank_a], xb = uniq[(int64_t)bf * n + br.rank_b];
    const double thr = split_threshold(xa, xb);
    const int32_t lraw = atomicAdd(&pool.nn[nd.b], 2);
    const int64_t r = (int64_t)nd.b * pool.cap;
    pool.feature[r + nd.raw] = bf;
    pool.thr[r + nd.raw] = thr;
    pool.left[r + nd.raw] = lraw;
    pool.drss[r + nd.raw] = ldexp(__ddiv_rn(bg, (double)nd.n), -2 * q);
    const uint32_t t = (uint32_t)(t0 + nd.b);
    cl.a = br.pos + 1;
    cl.n = br.nl;
    cl.S = br.Sl;
    cl.key = child_key(seed, t, nd.key, 0);
    cl.raw = lraw;
    cr.a = nd.a - cl.a;
    cr.n = nd.n - br.nl;
    cr.S = nd.S - br.Sl;
    cr.key = child_key(seed, t, nd.key, 1);
    cr.raw = lraw + 1;
    Child* cs[2] = {&cl, &cr};
    for (int side = 0; side < 2; ++side) {
      Child& c = *cs[side];
      c.base = 0;
      if (c.n <= nodesize || c.a < 2) c.kind = KIND_LEAF;
      else if (c.a <= Asmall) c.kind = KIND_SMALL;
      else c.kind = KIND_LARGE;
      pool.feature[r + c.raw] = -1;
      pool.left[r + c.raw] = -1;
      pool.count[r + c.raw] = c.n;
      pool.thr[r + c.raw] = 0.0;
      pool.drss[r + c.raw] = 0.0;
    }
    atomicAdd(&sum->split_a, (unsigned long long)nd.a);
    sp.split = 1;
    sp.f = bf;
    sp.pos = br.pos;
    sp.lraw = lraw;
    sp.nl = cl.n;
    sp.nr = cr.n;
  }
  split[k] = sp;
  child[2 * k] = cl;
  child[2 * k + 1] = cr;
  packL[2 * k] = cl.kind == KIND_LARGE ? (((uint64_t)cl.a << 32) | 1u) : 0ull;
  packL[2 * k + 1] = cr.kind == KIND_LARGE ? (((uint64_t)cr.a << 32) | 1u) : 0ull;
  packS[2 * k] = cl.kind == KIND_SMALL ? (((uint64_t)cl.a << 32) | 1u) : 0ull;
  packS[2 * k + 1] = cr.kind == KIND_SMALL ? (((uint64_t)cr.a << 32) | 1u) : 0ull;
}

// child placement: next-level node list and small queue
__global__ void k_child_place(int N2, int p, const LNode* nodes, Child* child, const uint64_t* scanL,
                              const uint64_t* scanS, LNode* next, LNode* sq, const LevelSummary* prev) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= N2) return;
  const Child ch = child[c];
  if (ch.kind != KIND_LARGE && ch.kind != KIND_SMALL) return;
  LNode nd;
  nd.b = nodes[c >> 1].b;
  nd.raw = ch.raw;
  nd.a = ch.a;
  nd.n = ch.n;
  nd.S = ch.S;
  nd.key = ch.key;
  if (ch.kind == KIND_LARGE) {
    const uint64_t sc = scanL[c];
    nd.base = (int64_t)p * (int64_t)(sc >> 32);
    child[c].base = nd.base;
    next[(uint32_t)sc] = nd;
  } else {
    const uint64_t sc = scanS[c];
    nd.base = prev->small_elems + (int64_t)p * (int64_t)(sc >> 32);
    child[c].base = nd.base;
    sq[prev->nsmall + (uint32_t)sc] = nd;
  }
}

__global__ void k_commit(int N2, const uint64_t* packL, const uint64_t* scanL, const uint64_t* packS,
                         const uint64_t* scanS, int p, LevelSummary* sum, LevelSummary* host_sum) {
  LevelSummary s = *sum;
  uint64_t tl = 0, ts = 0;
  if (N2 > 0) {
    tl = scanL[N2 - 1] + packL[N2 - 1];
    ts = scanS[N2 - 1] + packS[N2 - 1];
  }
  s.nnext = (int32_t)(uint32_t)tl;
  s.next_elems = (int64_t)p * (int64_t)(tl >> 32);
  s.nsmall += (int32_t)(uint32_t)ts;
  s.small_elems += (int64_t)p * (int64_t)(ts >> 32);
  *host_sum = s;
  s.split_a = 0;
  *sum = s;
}

// ------------------------------------------------------------------ pieces (goes-right flags)
// Every winning segment of a level is cut into pieces of PIECE entries; one
// CTA per piece (k_dest_bits).
constexpr int PIECE_V = 8;
constexpr int PIECE = NT * PIECE_V;  // 2048 entries

// items: mode 0 scan (node = i / mtry), 1 dest (node = i, split only), 2 partition (node = i / p, split with a kept child)
__global__ void k_piece_count(int mode, int nitems, int div, const LNode* nodes, const Split* split, const Child* child,
                              int32_t* cnt) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nitems) return;
  const int k = i / div;
  int a = nodes[k].a;
  if (mode >= 1 && !split[k].split) a = 0;
  if (mode == 2) {
    const int kl = child[2 * k].kind, kr = child[2 * k + 1].kind;
    if (kl != KIND_LARGE && kl != KIND_SMALL && kr != KIND_LARGE && kr != KIND_SMALL) a = 0;
  }
  cnt[i] = (a + PIECE - 1) / PIECE;
}

__global__ void k_piece_map(int nitems, const int32_t* cnt, const int32_t* off, int32_t* map, int32_t* total) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nitems) return;
  const int c = cnt[i], o = off[i];
  for (int k = 0; k < c; ++k) map[o + k] = i;
  if (i == nitems - 1) *total = o + c;
}

struct DestArgs {
  const LNode* nodes;
  const Split* split;
  const uint64_t* E;
  const double* y;
  int64_t n;
  uint8_t* side;
  const int32_t* poff;
  const int32_t* pmap;
  const int32_t* ptotal;
  double* csum;  // 2 per node: sum of w*y of the left / right child
};

__global__ void k_child_values(int N, const Split* split, const double* csum, const LNode* nodes, Pool pool) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= N) return;
  const Split sp = split[k];
  if (!sp.split) return;
  const int64_t r = (int64_t)nodes[k].b * pool.cap;
  pool.value[r + sp.lraw] = __ddiv_rn(csum[2 * k], (double)sp.nl);
  pool.value[r + sp.lraw + 1] = __ddiv_rn(csum[2 * k + 1], (double)sp.nr);
}

// ------------------------------------------------------------------ TMA bulk copies + read-only gathers (global phase)
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar)) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra WAIT_%=;\n}\n" ::"r"(
          smem_u32(bar)),
      "r"(phase)
      : "memory");
}
// Stage entries [src, src + cnt): the copy starts at the 16-byte aligned address at or below src;
// returns the entry offset (0 or 1) of src inside the buffer.  Issued by one thread.
__device__ __forceinline__ int stage_entries(uint64_t* buf, const uint64_t* src, int cnt, uint64_t* bar) {
  const uintptr_t a = (uintptr_t)src, a0 = a & ~(uintptr_t)15;
  const int off = (int)((a - a0) >> 3);
  const uint32_t bytes = (uint32_t)((((size_t)(cnt + off) * 8) + 15) & ~(size_t)15);
  tma_load_1d(buf, (const void*)a0, bytes, bar);
  return off;
}
// Gathers issued with volatile asm: ptxas keeps them back to back, so all of a
// thread's independent loads are in flight together (otherwise it converts each
// loaded value to a predicate at once and serialises the L2 round trips).
__device__ __forceinline__ uint32_t ldg_u8_nc(const uint8_t* p) {
  uint32_t v;
  asm volatile("ld.global.nc.u8 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint32_t ldg_u32_nc(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ int64_t ldg_s64_nc(const int64_t* p) {
  int64_t v;
  asm volatile("ld.global.nc.s64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ float rcp_approx(float x) {  // |rel err| < 2^-22
  float r;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
// Cheap rigorous bounds gL <= g <= gU of the S4.3 key (fp64, no int128).
__device__ __forceinline__ void key_bounds(double nkd, double Skd, int64_t nk, int32_t nl, int64_t Sl, double& gL,
                                           double& gU) {
  const double a = nkd * (double)Sl, b = (double)nl * Skd;
  const double d = fabs(a - b);
  const double E = (fabs(a) + fabs(b)) * 8.881784197001252e-16;  // 2^-50
  const double r = (double)rcp_approx((float)(nl * (nk - nl)));
  const double hi = (d + E), lo = fmax(d - E, 0.0);
  gU = hi * hi * r * (1.0 + 9.5367431640625e-07);  // (1 + 2^-20)
  gL = lo * lo * r * (1.0 - 9.5367431640625e-07);
}

// The same screen in fp32 on t = sqrt(g) = |D| / sqrt(n_l n_r) (monotone in the key, < 2^84 so no overflow):
// tL <= t <= tU rigorously.  a = RN32(n_k RN32(S_l)), b = RN32(n_l RN32(S_k)) each lie within 2^-23 (1 + 2^-23)
// of n_k S_l, n_l S_k, and RN32|a - b| within 2^-24 more, so |D| is within E = (|a| + |b|) 2^-21 of
// RN32|a - b|; the directed roundings and the (1 +- 2^-20) factors absorb rsqrtf's error (< 2^-22) and make
// tU >= t (1 + 2^-21), tL <= t (1 - 2^-21): a candidate screened out (tU < M) has a key below every key
// that reaches M by a relative 2^-19, so it can neither beat nor tie it.
__device__ __forceinline__ void key_bounds_t(float nkf, float Skf, int64_t nk, int32_t nl, int64_t Sl, float& tL,
                                             float& tU) {
  const float a = nkf * __ll2float_rn(Sl), b = __int2float_rn(nl) * Skf;
  const float d = fabsf(a - b);
  const float E = (fabsf(a) + fabsf(b)) * 4.76837158203125e-07f;  // 2^-21
  const float hi = __fadd_ru(d, E), lo = fmaxf(__fsub_rd(d, E), 0.0f);
  const float nlf = __int2float_rn(nl), nrf = __ll2float_rn(nk - nl);  // exact: < 2^24
  tU = __fmul_ru(__fmul_ru(hi, rsqrtf(__fmul_rd(nlf, nrf))), 1.00000095367431640625f);  // (1 + 2^-20)
  tL = __fmul_rd(__fmul_rd(lo, rsqrtf(__fmul_ru(nlf, nrf))), 0.99999904632568359375f);  // (1 - 2^-20)
}
// A lower bound of t for an exact key g (the running best): sqrt(g) (1 - 2^-20), rounded down; -1 for none.
__device__ __forceinline__ float key_t_lower(double g) {
  return g >= 0.0 ? __fmul_rd(__fsqrt_rd(__double2float_rd(g)), 0.99999904632568359375f) : -1.0f;
}
// Warp max of non-negative floats (-1 = none) through their bit patterns.
__device__ __forceinline__ float warp_max_t(float v) {
  const uint32_t k = v >= 0.0f ? __float_as_uint(v) + 1u : 0u;
  const uint32_t m = __reduce_max_sync(0xffffffffu, k);
  return m ? __uint_as_float(m - 1u) : -1.0f;
}

// ------------------------------------------------------------------ tree-affine item kernels (global phase v6)
// Nodes of a level are ordered by tree, so each tree's items (node, feature)
// form a contiguous range.  A CTA is bound to one tree and owns whole items
// (round robin over the tree's items): it walks an item unit by unit with a
// running carry -- no cross-CTA prefix, no look-back, no extra pass -- and the
// bulk copy (TMA) of its next unit is in flight while it works on the current
// one.  The partition kernel keeps the tree's goes-right bitmap (n bits) in
// shared memory, so the per-entry side lookup is a shared-memory bit test.
__global__ void k_tree_ranges(int N, const LNode* nodes, int32_t* lo, int32_t* hi) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= N) return;
  const int b = nodes[k].b;
  if (k == 0 || nodes[k - 1].b != b) lo[b] = k;
  if (k == N - 1 || nodes[k + 1].b != b) hi[b] = k + 1;
}

// The level's trees that have nodes (thi > tlo), in tree order; one CTA of >= B threads.
__global__ void k_active_trees(int B, const int32_t* tlo, const int32_t* thi, int32_t* active, int32_t* nactive) {
  __shared__ int32_t cnt;
  if (threadIdx.x == 0) cnt = 0;
  __syncthreads();
  for (int b0 = 0; b0 < B; b0 += blockDim.x) {
    const int b = b0 + threadIdx.x;
    const bool on = b < B && thi[b] > tlo[b];
    const unsigned m = __ballot_sync(0xffffffffu, on);
    __shared__ int32_t wbase[32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (lane == 0) wbase[wid] = __popc(m);
    __syncthreads();
    if (threadIdx.x == 0) {
      int run = cnt;
      for (int w = 0; w < (int)(blockDim.x >> 5); ++w) {
        const int c = wbase[w];
        wbase[w] = run;
        run += c;
      }
      cnt = run;
    }
    __syncthreads();
    if (on) active[wbase[wid] + __popc(m & ((1u << lane) - 1u))] = b;
    __syncthreads();
  }
  if (threadIdx.x == 0) *nactive = cnt;
}

struct TreeSched {  // CTA -> (tree, slot, slots per tree)
  int b0, bstep, c, C;
};
__device__ __forceinline__ TreeSched tree_sched(int B) {
  const int G = gridDim.x, gi = blockIdx.x;
  TreeSched s;
  if (G >= B) {
    s.b0 = gi % B;
    s.bstep = B;  // single tree
    s.c = gi / B;
    s.C = G / B + (s.b0 < G % B ? 1 : 0);
  } else {
    s.b0 = gi;
    s.bstep = G;
    s.c = 0;
    s.C = 1;
  }
  return s;
}

struct TScanArgs {
  const LNode* nodes;
  const int32_t* feat;
  int mtry, B;
  const uint64_t* E;
  const int64_t* yq;
  const int32_t* tlo;  // per tree: first node of the level (or 0) / one past the last
  const int32_t* thi;
  Rec* rec;
  const int32_t* active;   // the level's trees that have nodes, and how many (k_active_trees)
  const int32_t* nactive;
};

constexpr int SNT = 128;            // threads of the split-scan CTA (4 CTAs per SM: independent unit pipelines)
// entries per thread: 9 (odd: conflict-free 64-bit shared loads; 1152-entry units, 9 KB bulk copies); measured:
// 64 threads / 7 or 13 entries slower

// The exact key off the unrolled scan loops (rarely reached: only where the upper bound passes the screen).
__device__ __noinline__ double split_key_call(int64_t nk, int64_t Sk, int64_t nl, int64_t Sl) {
  return split_key(nk, Sk, nl, Sl);
}

struct WBest {  // best exact candidate of one warp for the current unit
  double g;
  uint32_t rank, rb;
  int32_t pos, nl;
  int64_t Sl;
};

// a7 split search: one CTA owns whole (node, drawn feature) items of one tree.
// Per unit (TMA bulk copy, double-buffered): each thread takes TSV consecutive
// entries, gathers y_q[row] (all TSV in flight), scans serially in registers on
// top of ONE block scan of (n, S); every boundary gets cheap rigorous bounds
// gL <= g <= gU (fp64), the unit's threshold M = max(best gL, item best) is one
// block max, and only boundaries with gU >= M get the exact S4.3 key.  Four
// barriers per unit; each thread re-derives the block results from the
// per-warp values, so there are no broadcast round trips.
// TSV entries per thread (unit = SNT * TSV entries), MINB CTAs per SM for the register budget (BF_SCAN_TSV: 9 default)
template <int TSV, int MINB>
__global__ void __launch_bounds__(SNT, MINB) k_split_scan_tree(TScanArgs g) {
  constexpr int TUNIT = SNT * TSV;
  extern __shared__ __align__(16) unsigned char dsm[];
  uint64_t* bufs = (uint64_t*)dsm;  // 2 x (TUNIT + 4)
  constexpr int NW = SNT / 32;
  __shared__ uint64_t bar[2];
  __shared__ int32_t smc[NW];
  __shared__ int64_t sms[NW];
  __shared__ float smL[NW];
  __shared__ WBest swb[NW];
  __shared__ int s_off[2];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  // CTAs are spread over the level's ACTIVE trees (deep levels often have nodes in a few trees only)
  const int NA = *g.nactive;
  const TreeSched ts = tree_sched(NA);
  if (tid == 0) {
    mbar_init(&bar[0]);
    mbar_init(&bar[1]);
  }
  __syncthreads();
  uint32_t phase[2] = {0u, 0u};
  int cur = 0;
  for (int ai = ts.b0; ai < NA; ai += ts.bstep) {
    const int b = g.active[ai];
    const int i_lo = g.tlo[b] * g.mtry, i_hi = g.thi[b] * g.mtry;
    int item = i_lo + ts.c, unit = 0;
    auto issue = [&](int it, int un, int slot) {
      const LNode nd = g.nodes[it / g.mtry];
      const int f = g.feat[it];
      const int u0 = un * TUNIT;
      const int cload = min(TUNIT + 1, nd.a - u0);
      s_off[slot] = stage_entries(bufs + (size_t)slot * (TUNIT + 4), g.E + nd.base + (int64_t)f * nd.a + u0, cload,
                                  &bar[slot]);
    };
    if (item >= i_hi) continue;
    if (tid == 0) issue(item, 0, cur);
    // running state of the current item (identical in every thread)
    int32_t carry_n = 0;
    int64_t carry_S = 0;
    WBest ib;
    ib.g = -1.0;
    ib.rank = 0xffffffffu;
    ib.rb = 0;
    ib.pos = -1;
    ib.nl = 0;
    ib.Sl = 0;
    LNode nd = g.nodes[item / g.mtry];
    while (item < i_hi) {
      const int nun = (nd.a + TUNIT - 1) / TUNIT;
      int nitem = item, nunit = unit + 1;
      if (nunit >= nun) {
        nitem = item + ts.C;
        nunit = 0;
      }
      __syncthreads();  // S0: the other buffer and the per-warp slots are free
      if (tid == 0 && nitem < i_hi) issue(nitem, nunit, cur ^ 1);
      const int a = nd.a, u0 = unit * TUNIT, cnt = min(TUNIT, a - u0);
      const int64_t nk = nd.n, Sk = nd.S;
      const float nkf = __ll2float_rn(nk), Skf = __ll2float_rn(Sk);  // nk < 2^24: exact
      mbar_wait(&bar[cur], phase[cur]);
      phase[cur] ^= 1u;
      const uint64_t* buf = bufs + (size_t)cur * (TUNIT + 4) + s_off[cur];
      const int jl = tid * TSV;
      // the thread's entries, read from shared memory once: rank (and the next entry's), w, w * y_q
      uint32_t rk[TSV + 1];
      int32_t wq[TSV];
      int64_t wy[TSV];
#pragma unroll
      for (int q = 0; q < TSV; ++q) {
        const bool in = jl + q < cnt;
        const uint64_t e = buf[min(jl + q, cnt)];  // buf[cnt]: the next unit's first entry (if any)
        rk[q] = e_rank(e);
        wq[q] = in ? e_w(e) : 0;
        wy[q] = ldg_s64_nc(g.yq + (in ? e_row(e) : 0u));
      }
      rk[TSV] = e_rank(buf[min(jl + TSV, cnt)]);  // the entry after my last (checked against a below)
      int32_t tc = 0;
      int64_t tsum = 0;
#pragma unroll
      for (int q = 0; q < TSV; ++q) {
        wy[q] *= wq[q];
        tc += wq[q];
        tsum += wy[q];
      }
      // S1: one block scan of (n, S): warp inclusive scans, per-warp totals, every thread adds the earlier warps'
      int32_t ic = tc;
      int64_t is = tsum;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int32_t uc = __shfl_up_sync(0xffffffffu, ic, o);
        const int64_t us = __shfl_up_sync(0xffffffffu, is, o);
        if (lane >= o) {
          ic += uc;
          is += us;
        }
      }
      if (lane == 31) {
        smc[wid] = ic;
        sms[wid] = is;
      }
      __syncthreads();
      int32_t prc0 = carry_n + ic - tc, totc = 0;
      int64_t prs0 = carry_S + is - tsum, tots = 0;
#pragma unroll
      for (int k = 0; k < NW; ++k) {
        const int32_t c = smc[k];
        const int64_t v = sms[k];
        if (k < wid) {
          prc0 += c;
          prs0 += v;
        }
        totc += c;
        tots += v;
      }
      // bounds of every boundary (fp32, t = sqrt(key) space); the thread's best lower bound
      float gUf[TSV];
      float mL = key_t_lower(ib.g);
      {
        int32_t prc = prc0;
        int64_t prs = prs0;
#pragma unroll
        for (int q = 0; q < TSV; ++q) {
          gUf[q] = -1.0f;
          const int j = jl + q;
          if (j < cnt) {
            prc += wq[q];
            prs += wy[q];
            if (u0 + j + 1 < a && rk[q] != rk[q + 1]) {
              float tL, tU;
              key_bounds_t(nkf, Skf, nk, prc, prs, tL, tU);
              mL = fmaxf(mL, tL);
              gUf[q] = tU;
            }
          }
        }
      }
      // S2: block max of the lower bounds -> M
      {
        const float wm = warp_max_t(mL);
        if (lane == 0) smL[wid] = wm;
      }
      __syncthreads();
      float M = -1.0f;
#pragma unroll
      for (int k = 0; k < NW; ++k) M = fmaxf(M, smL[k]);
      // exact keys where the upper bound reaches M
      WBest tb;
      tb.g = -1.0;
      tb.rank = 0xffffffffu;
      tb.rb = 0;
      tb.pos = -1;
      tb.nl = 0;
      tb.Sl = 0;
      {
        int32_t prc = prc0;
        int64_t prs = prs0;
#pragma unroll
        for (int q = 0; q < TSV; ++q) {
          const int j = jl + q;
          if (j < cnt) {
            prc += wq[q];
            prs += wy[q];
            if (gUf[q] >= M && gUf[q] >= 0.0f) {
              const double gk = split_key_call(nk, Sk, prc, prs);
              const uint32_t ra = rk[q];
              if (rec_better(gk, ra, tb.g, tb.rank)) {
                tb.g = gk;
                tb.rank = ra;
                tb.rb = rk[q + 1];
                tb.pos = u0 + j;
                tb.nl = prc;
                tb.Sl = prs;
              }
            }
          }
        }
      }
      // the warp's winner of the unit merges into the warp's running best (no block barrier per unit: every
      // warp's best is an exact candidate key, so the block max of the lower bounds above still screens
      // correctly); the warps' bests are merged once per item
      {
        const int wl = warp_argmax_key(gkey(tb.g), tb.rank);
        if (wl >= 0) {
          WBest wb;
          wb.g = __shfl_sync(0xffffffffu, tb.g, wl);
          wb.rank = __shfl_sync(0xffffffffu, tb.rank, wl);
          wb.rb = __shfl_sync(0xffffffffu, tb.rb, wl);
          wb.pos = __shfl_sync(0xffffffffu, tb.pos, wl);
          wb.nl = __shfl_sync(0xffffffffu, tb.nl, wl);
          wb.Sl = __shfl_sync(0xffffffffu, tb.Sl, wl);
          if (wb.g > ib.g || (wb.g == ib.g && wb.rank < ib.rank)) ib = wb;
        }
      }
      carry_n += totc;
      carry_S += tots;
      if (unit + 1 >= nun) {  // item done: merge the warps' bests (position order == rank order)
        if (lane == 0) swb[wid] = ib;
        __syncthreads();
        if (tid == 0) {
          WBest bb = swb[0];
#pragma unroll
          for (int k = 1; k < NW; ++k) {
            const WBest& o = swb[k];
            if (o.g >= 0.0 && (o.g > bb.g || (o.g == bb.g && o.rank < bb.rank))) bb = o;
          }
          Rec R;
          R.g = bb.g;
          R.rank_a = bb.rank;
          R.rank_b = bb.rb;
          R.pos = bb.pos;
          R.nl = bb.nl;
          R.Sl = bb.Sl;
          g.rec[item] = R;
        }
        carry_n = 0;
        carry_S = 0;
        ib.g = -1.0;
        ib.rank = 0xffffffffu;
        ib.rb = 0;
        ib.pos = -1;
        ib.nl = 0;
        ib.Sl = 0;
        if (nitem < i_hi) nd = g.nodes[nitem / g.mtry];
      }
      item = nitem;
      unit = nunit;
      cur ^= 1;
    }
  }
}

struct TPartArgs {
  const LNode* nodes;
  const Split* split;
  const Child* child;
  int p, B;
  const uint64_t* Ecur;
  const uint32_t* sideb;  // per tree: n bits, 1 = goes right
  int64_t nw;             // words per tree
  int bitmap_smem;        // 1: stage the tree's bitmap in shared memory
  uint64_t* Enext;
  uint64_t* Esmall;
  const int32_t* tlo;
  const int32_t* thi;
  const int32_t* ioff;  // per node: first work item (N + 1 entries; items of a tree are contiguous)
  const int2* imap;     // per work item: (node, first feature)
  const int32_t* active;   // the level's trees that have nodes, and how many (k_active_trees)
  const int32_t* nactive;
};

constexpr int TPNT = 512;           // threads of the partition CTA (one CTA per SM: the bitmap fills shared memory)
constexpr int TPG = 2;              // independent unit pipelines per CTA (thread groups sharing the bitmap)
constexpr int TPGT = TPNT / TPG;    // threads per group
constexpr int TPV = 7;
constexpr int TPUNIT = TPGT * TPV;  // 1792 entries per unit
constexpr int TPNS = 2;             // bulk-copy buffers per group (units in flight: TPNS - 1 ahead; 3 measured slower)

__device__ __forceinline__ bool part_item_active(const Split* split, const Child* child, int node) {
  if (!split[node].split) return false;
  const int kl = child[2 * node].kind, kr = child[2 * node + 1].kind;
  return kl == KIND_LARGE || kl == KIND_SMALL || kr == KIND_LARGE || kr == KIND_SMALL;
}

// Features per work item: an item is a contiguous range of the node's block (its feature segments are
// contiguous, and every segment has exactly al lefts), so the item is stable-partitioned as ONE stream with a
// running left count: lefts land at f0 * al + (lefts so far), rights at f0 * ar + (rights so far).  Items of
// about PART_ITEM_UNITS units keep the units full (only an item's last unit is partial).
constexpr int PART_ITEM_UNITS = 16;
__host__ __device__ __forceinline__ int part_group(int a, int p) {
  const int tgt = PART_ITEM_UNITS * TPUNIT;
  return a >= tgt ? 1 : min(p, tgt / a);
}

// Work items of the partition (node, group of consecutive features), listed per level so that a
// partition CTA finds its next item with one load instead of walking the tree's item sequence.
__global__ void k_part_items_count(int N, int p, const LNode* nodes, const Split* split, const Child* child,
                                   int32_t* cnt) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k > N) return;
  int c = 0;
  if (k < N && part_item_active(split, child, k)) c = (p + part_group(nodes[k].a, p) - 1) / part_group(nodes[k].a, p);
  cnt[k] = c;
}
__global__ void k_part_items_map(int N, int p, const LNode* nodes, const int32_t* cnt, const int32_t* off, int2* map) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= N) return;
  const int c = cnt[k], o = off[k], gsz = part_group(nodes[k].a, p);
  for (int i = 0; i < c; ++i) map[o + i] = make_int2(k, i * gsz);
}

// a9 partition: one CTA owns whole work items of one tree; lefts first, stable.
// A work item is (node, group of G consecutive features), G = part_group(a, p):
// a contiguous range of the node's block, walked in full units of TPUNIT
// entries (bulk copies that may straddle feature segments) with a running left
// count; the left (right) outputs of consecutive features are contiguous in
// the child's block, so the group partitions as one stream.
struct PWork {
  int node, f0, g, unit;  // node index, first feature, features in the item, unit index inside the item
  int a, nun;             // the node's entries per feature; units of the item
  int64_t base;
  int kl, al, kr, ar;     // children: kind and entries per feature
  int64_t bl, br;         // children: block offsets
};

// Group-local barrier (named barrier 1 + group over the group's TPGT threads).
__device__ __forceinline__ void group_sync(int grp) {
  asm volatile("bar.sync %0, %1;" ::"r"(1 + grp), "r"(TPGT) : "memory");
}
// The CTA's TPG thread groups share the tree's goes-right bitmap in shared memory and run independent unit
// pipelines (own bulk-copy buffers, mbarriers and named barriers) over alternate items of the CTA's slice,
// so one group's barrier and copy waits overlap the other group's work.
__global__ void __launch_bounds__(TPNT) k_partition_tree(TPartArgs g) {
  extern __shared__ __align__(16) unsigned char dsm[];
  const int tid = threadIdx.x, grp = tid / TPGT, lt = tid % TPGT;
  uint64_t* gbase = (uint64_t*)dsm + (size_t)grp * (TPNS * (TPUNIT + 2));
  uint64_t* bufs = gbase;                       // TPNS x (TPUNIT + 2): bulk-copy ring, TPNS - 1 units ahead
  uint32_t* bm = (uint32_t*)((uint64_t*)dsm + (size_t)TPG * (TPNS * (TPUNIT + 2)));  // nw words (if staged)
  __shared__ uint64_t bars[TPG][TPNS];
  __shared__ int32_t sms[TPG][TPGT / 32];
  __shared__ int s_offs[TPG][TPNS];
  __shared__ PWork s_ws[TPG][TPNS];
  uint64_t* bar = bars[grp];
  int32_t* sm = sms[grp];
  int* s_off = s_offs[grp];
  PWork* s_w = s_ws[grp];
  const int NA = *g.nactive;  // CTAs spread over the level's active trees
  const TreeSched ts = tree_sched(NA);
  if (lt == 0)
    for (int k = 0; k < TPNS; ++k) mbar_init(&bar[k]);
  __syncthreads();
  uint32_t phase[TPNS] = {};
  int cur = 0;
  for (int ai = ts.b0; ai < NA; ai += ts.bstep) {
    const int b = g.active[ai];
    const int n_lo = g.tlo[b], n_hi = g.thi[b];
    if (n_lo >= n_hi) continue;
    const uint32_t* sideg = g.sideb + (int64_t)b * g.nw;
    __syncthreads();  // both groups are done with the previous tree's bitmap
    if (g.bitmap_smem)
      for (int64_t w = tid; w < g.nw; w += TPNT) bm[w] = sideg[w];
    __syncthreads();
    const uint32_t* sb = g.bitmap_smem ? bm : sideg;
    // this group's work items of the tree: the CTA takes every C-th item of the tree's contiguous item range
    // (k_part_items_*), its groups alternate; an owned item yields all its units in order (the running left
    // count stays inside one group)
    const int step = ts.C * TPG;
    int jcur = g.ioff[n_lo] + ts.c + grp * ts.C;
    const int jend = g.ioff[n_hi];
    // the group's thread 0 walks the items; the map entry of the next item is loaded one item ahead and its
    // node / children records (and the map entry after it) are prefetched into L1
    auto pf = [&](const void* ptr) { asm volatile("prefetch.global.L1 [%0];" ::"l"(ptr)); };
    auto pf_item = [&](int2 it) {
      pf(g.nodes + it.x);
      pf(g.child + 2 * it.x);
    };
    int2 nxt = make_int2(-1, 0);
    if (lt == 0 && jcur < jend) {
      nxt = g.imap[jcur];
      pf_item(nxt);
      if (jcur + step < jend) pf(g.imap + jcur + step);
    }
    PWork cw;
    cw.nun = 0;
    int cur_unit = 0;  // next unit of the owned item being emitted
    auto next_mine = [&](PWork& w) -> bool {
      if (cur_unit < cw.nun) {
        w = cw;
        w.unit = cur_unit++;
        return true;
      }
      if (jcur >= jend) return false;
      const int2 it = nxt;
      jcur += step;
      if (jcur < jend) {
        nxt = g.imap[jcur];
        pf_item(nxt);
        if (jcur + step < jend) pf(g.imap + jcur + step);
      }
      const LNode nd = g.nodes[it.x];
      const Child c0 = g.child[2 * it.x], c1 = g.child[2 * it.x + 1];
      cw.node = it.x;
      cw.f0 = it.y;
      cw.a = nd.a;
      cw.base = nd.base;
      cw.g = min(part_group(nd.a, g.p), g.p - it.y);
      cw.nun = (int)(((int64_t)cw.g * nd.a + TPUNIT - 1) / TPUNIT);
      cw.unit = 0;
      cw.kl = c0.kind;
      cw.al = c0.a;
      cw.bl = c0.base;
      cw.kr = c1.kind;
      cw.ar = c1.a;
      cw.br = c1.base;
      cur_unit = 1;
      w = cw;
      return true;
    };
    auto issue = [&](const PWork& w, int slot) {
      const int u0 = w.unit * TPUNIT;
      const int cnt = min(TPUNIT, w.g * w.a - u0);
      s_off[slot] = stage_entries(bufs + (size_t)slot * (TPUNIT + 2), g.Ecur + w.base + (int64_t)w.f0 * w.a + u0, cnt,
                                  &bar[slot]);
    };
    // the group's thread 0 runs the item pipeline TPNS - 1 units ahead and publishes each unit's record in s_w
    if (lt == 0) {
      bool more = true;
      for (int k = 0; k + 1 < TPNS; ++k) {
        PWork w0;
        if (!more || !next_mine(w0)) {
          w0.node = -1;
          more = false;
        }
        const int sl = (cur + k) % TPNS;
        s_w[sl] = w0;
        if (w0.node >= 0) issue(w0, sl);
      }
    }
    group_sync(grp);
    if (s_w[cur].node < 0) continue;
    int64_t carry_l = 0;
    for (;;) {
      group_sync(grp);  // the buffer and s_w slot of unit k - 1 are free
      const PWork w = s_w[cur];
      if (w.node < 0) break;
      const int nxt = (cur + 1) % TPNS;
      if (lt == 0) {
        const int sl = (cur + TPNS - 1) % TPNS;  // unit k + TPNS - 1
        PWork wn;
        if (s_w[(cur + TPNS - 2) % TPNS].node < 0 || !next_mine(wn)) wn.node = -1;
        s_w[sl] = wn;
        if (wn.node >= 0) issue(wn, sl);
      }
      const int a = w.a;
      const int u0 = w.unit * TPUNIT;
      const int cnt = min(TPUNIT, w.g * a - u0);
      mbar_wait(&bar[cur], phase[cur]);
      phase[cur] ^= 1u;
      const uint64_t* buf = bufs + (size_t)cur * (TPUNIT + 2) + s_off[cur];
      // Warp wg of the group owns the unit's entries [wg * 32 TPV, (wg + 1) * 32 TPV), read striped (entry
      // wg * 32 TPV + 32 q + lane): per round q the lanes' lefts (rights) are consecutive in the output, so each
      // store instruction writes one contiguous run straight to the child block in global memory -- no shared
      // staging buffer, one group barrier per unit for the warps' left counts.
      const int lane = lt & 31, wg = lt >> 5;
      const int wb0 = wg * (TPV * 32);
      uint64_t ev[TPV];
      uint32_t bw[TPV];
#pragma unroll
      for (int q = 0; q < TPV; ++q) ev[q] = buf[min(wb0 + 32 * q + lane, cnt - 1)];
      if (g.bitmap_smem) {
#pragma unroll
        for (int q = 0; q < TPV; ++q) bw[q] = sb[e_row(ev[q]) >> 5];
      } else {  // L2-resident bitmap: all gathers in flight together
#pragma unroll
        for (int q = 0; q < TPV; ++q) bw[q] = ldg_u32_nc(sb + (e_row(ev[q]) >> 5));
      }
      uint32_t lmk[TPV];
      int32_t wl_cnt = 0;
#pragma unroll
      for (int q = 0; q < TPV; ++q) {
        const bool left = wb0 + 32 * q + lane < cnt && !((bw[q] >> (e_row(ev[q]) & 31)) & 1u);
        lmk[q] = __ballot_sync(0xffffffffu, left);
        wl_cnt += __popc(lmk[q]);
      }
      if (lane == 0) sm[wg] = wl_cnt;
      group_sync(grp);
      int32_t preL = 0, tot = 0;
#pragma unroll
      for (int k = 0; k < TPGT / 32; ++k) {
        const int32_t v = sm[k];
        if (k < wg) preL += v;
        tot += v;
      }
      const int al = w.al, ar = w.ar;  // lefts / rights per feature segment
      const bool keepL = w.kl == KIND_LARGE || w.kl == KIND_SMALL;
      const bool keepR = w.kr == KIND_LARGE || w.kr == KIND_SMALL;
      const int64_t exl = carry_l, exr = (int64_t)u0 - carry_l;
      uint64_t* dl = (w.kl == KIND_LARGE ? g.Enext : g.Esmall) + w.bl + (int64_t)w.f0 * al + exl + preL;
      uint64_t* dr = (w.kr == KIND_LARGE ? g.Enext : g.Esmall) + w.br + (int64_t)w.f0 * ar + exr +
                     (min(wb0, cnt) - preL);
      const uint32_t ltm = (1u << lane) - 1u;
      int runL = 0, runR = 0;
#pragma unroll
      for (int q = 0; q < TPV; ++q) {
        const int j = wb0 + 32 * q + lane;
        const uint32_t vm = __ballot_sync(0xffffffffu, j < cnt);
        const uint32_t rm = vm & ~lmk[q];
        if ((lmk[q] >> lane) & 1u) {
          if (keepL) dl[runL + __popc(lmk[q] & ltm)] = ev[q];
        } else if ((rm >> lane) & 1u) {
          if (keepR) dr[runR + __popc(rm & ltm)] = ev[q];
        }
        runL += __popc(lmk[q]);
        runR += __popc(rm);
      }
      carry_l += tot;
      {
        const PWork& wn = s_w[nxt];  // published a unit ago
        if (wn.node != w.node || wn.f0 != w.f0) carry_l = 0;
      }
      cur = nxt;
    }
  }
}

// goes-right bitmap of the rows of every split node (from its winning segment) + child sums of w*y
__global__ void __launch_bounds__(NT) k_dest_bits(DestArgs g, uint32_t* sideb, int64_t nw) {
  __shared__ double sl[NT / 32], sr[NT / 32];
  const int t = blockIdx.x;
  if (t >= *g.ptotal) return;
  const int k = g.pmap[t], pc = t - g.poff[k];
  const Split sp = g.split[k];
  const LNode nd = g.nodes[k];
  const uint64_t* seg = g.E + nd.base + (int64_t)sp.f * nd.a;
  uint32_t* sb = sideb + (int64_t)nd.b * nw;
  double accl = 0.0, accr = 0.0;
  const int j0 = pc * PIECE + threadIdx.x * PIECE_V;
  uint64_t ev[PIECE_V];
  double yv[PIECE_V];
#pragma unroll
  for (int u = 0; u < PIECE_V; ++u) ev[u] = seg[min(j0 + u, nd.a - 1)];
#pragma unroll
  for (int u = 0; u < PIECE_V; ++u) yv[u] = __ldg(g.y + e_row(ev[u]));
#pragma unroll
  for (int u = 0; u < PIECE_V; ++u) {
    const int j = j0 + u;
    if (j < nd.a) {
      const uint32_t row = e_row(ev[u]);
      const int s = j > sp.pos;
      if (s) atomicOr(&sb[row >> 5], 1u << (row & 31));  // the level's bitmap starts cleared
      const double v = __dmul_rn((double)e_w(ev[u]), yv[u]);
      if (s) accr += v;
      else accl += v;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    accl += __shfl_down_sync(0xffffffffu, accl, o);
    accr += __shfl_down_sync(0xffffffffu, accr, o);
  }
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (lane == 0) {
    sl[wid] = accl;
    sr[wid] = accr;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double a0 = 0.0, a1 = 0.0;
    for (int q = 0; q < NT / 32; ++q) {
      a0 += sl[q];
      a1 += sr[q];
    }
    atomicAdd(&g.csum[2 * k], a0);
    atomicAdd(&g.csum[2 * k + 1], a1);
  }
}

// ------------------------------------------------------------------ subtree phase (one CTA per small node)
// Layout: the subtree's rows occupy local ids 0..a0-1.  list[f][0..a0) holds
// feature f's entries ((local rank << 16) | local row) sorted by value.  A
// MEDIUM node (a > TINY) owns the same column range [lo, lo+a) in every
// feature row; its split partitions each row's range in place (left part
// first), so children ranges nest.  A TINY root (a <= TINY) keeps its range
// [rlo, rlo+ra); its descendants are bit masks over the root's rows (bit =
// index of the row inside the root), evaluated by one warp with lane k
// holding the k-th entry of the root's sorted segment -- the node's rows in
// feature order are the lanes whose row bit is set, so no per-node sort or
// list partition is needed.  Tiny nodes go through a CTA-wide work queue so
// every warp stays busy until the whole subtree is grown.
constexpr int TINY = 64;
constexpr int MAXR = 32;  // small roots packed into one subtree CTA (their distinct rows add up to <= A)
constexpr int HBITS = 12, HSLOTS = 1 << HBITS;  // load-phase hash table (global row -> local id), a0 <= 1024
constexpr int TGRP = 7;   // drawn predictors staged per group in the tiny path
constexpr int TPU = 4;    // scan passes interleaved in the tiny path

struct SRec {  // node record of a subtree (local ids); thr is computed at flush from rows (ra, rb)
  int32_t feature, left, count;
  uint16_t ra, rb;
  double value, drss;
};
struct MNode {  // medium node (a > TINY) of a subtree level
  int32_t lo, a, n, id;
  int64_t S;
  uint64_t key;
  int32_t split, lid, al, nl;
  int64_t Sl;
  uint64_t keyl, keyr;
  int32_t kind[2];
};
template <int NWD>
struct TNodeT {  // tiny node: mask (NWD 64-bit words) over the rows of its tiny root [rlo, rlo+ra)
  int32_t rlo, ra;
  uint64_t mask[NWD];
  int32_t id;
  int32_t n;
  int64_t S;
  uint64_t key;
  double value;  // node value (S4.7): the warp that grows the node writes its whole record
};

// Row masks of tiny nodes (bit i = the row at feature-0 position i of the tiny root), 1 or 2 words; no dynamic
// indexing of the word array (it stays in registers).
template <int NWD>
__device__ __forceinline__ int m_popc(const uint64_t (&m)[NWD]) {
  int c = __popcll(m[0]);
  if constexpr (NWD == 2) c += __popcll(m[1]);
  return c;
}
template <int NWD>
__device__ __forceinline__ bool m_test(const uint64_t (&m)[NWD], int i) {
  if constexpr (NWD == 1) return (m[0] >> i) & 1ull;
  else return ((i < 64 ? m[0] : m[1]) >> (i & 63)) & 1ull;
}
template <int NWD>
__device__ __forceinline__ void m_set(uint64_t (&m)[NWD], int i) {
  if constexpr (NWD == 1) m[0] |= 1ull << i;
  else {
    const uint64_t b = 1ull << (i & 63);
    m[0] |= i < 64 ? b : 0ull;
    m[1] |= i < 64 ? 0ull : b;
  }
}
template <int NWD>
__device__ __forceinline__ void m_full(uint64_t (&m)[NWD], int a) {  // bits [0, a)
  m[0] = a >= 64 ? ~0ull : ((1ull << a) - 1ull);
  if constexpr (NWD == 2) m[1] = a >= 128 ? ~0ull : (a <= 64 ? 0ull : ((1ull << (a - 64)) - 1ull));
}
// index of the lowest set bit, which is cleared (0 for an empty mask)
template <int NWD>
__device__ __forceinline__ int m_pop(uint64_t (&m)[NWD]) {
  if constexpr (NWD == 1) {
    const int b = __ffsll((long long)m[0]) - 1;
    m[0] &= m[0] - 1;
    return b < 0 ? 0 : b;
  } else {
    const bool lo = m[0] != 0;
    const uint64_t v = lo ? m[0] : m[1];
    const int b = __ffsll((long long)v) - 1;
    const uint64_t v2 = v & (v - 1);
    m[0] = lo ? v2 : m[0];
    m[1] = lo ? m[1] : v2;
    return b < 0 ? 0 : b + (lo ? 0 : 64);
  }
}

struct WRec {  // best candidate found by one warp for its share of a node's features
  double g;
  int32_t f;
  uint32_t lrank;
  int32_t pos, nl;
  int64_t Sl;
  uint32_t ra, rb;
};

__host__ __device__ inline size_t align16(size_t x) { return (x + 15) & ~size_t(15); }
__host__ __device__ inline int max_medium(int A) { return A / (TINY + 1) + 2; }
__host__ __device__ inline int sub_temp(int A) { return A > TGRP * TINY ? A : TGRP * TINY; }
// The per-warp scratch area (medium partition temp / tiny staging of the TV = 0 path); in the tiny phase of the
// TV = 1 path it holds the position table ppos (p x A bytes), so it is sized for both.
__host__ __device__ inline size_t sub_temp_bytes(int A, int p) {
  const size_t a = (size_t)SUB_NW * sub_temp(A) * 4, b = (size_t)p * A;
  return a > b ? a : b;
}
static_assert(HSLOTS * 6 <= SUB_NW * TGRP * TINY * 4, "the load-phase hash table must fit the scratch area");

__host__ __device__ inline size_t subtree_smem(int A, int p, int tt = 64) {
  size_t s = 0;
  s += align16((size_t)p * A * 4);                    // list
  s += align16(sub_temp_bytes(A, p));                 // per-warp partition temp / tiny staging / ppos
  s += align16((size_t)A * 8) * 2;                    // wy, w*y
  s += align16((size_t)A * 4) * 2;                    // w, global row
  s += align16((size_t)A) * 2;                        // side, row index inside its tiny root
  s += align16((size_t)2 * A * sizeof(SRec));         // node records
  s += align16((size_t)2 * A * 2);                    // per record: tiny root of a deferred value (or 0xffff)
  s += align16((size_t)2 * max_medium(A) * sizeof(MNode));
  s += align16((size_t)(A + MAXR) * (tt > 64 ? sizeof(TNodeT<2>) : sizeof(TNodeT<1>)));   // tiny work queue
  s += align16((size_t)(A + MAXR) * 4);               // its ready flags
  s += align16((size_t)SUB_NW * p * 2) * 2;           // Fisher-Yates scratch, drawn features
  s += align16((size_t)SUB_NW * sizeof(WRec));
  s += 64;
  return s;
}

struct SubArgs {
  const LNode* sq;
  const int32_t* gperm;   // small roots in packing order (indices into sq)
  const int32_t* gstart;  // CTA g grows the roots gperm[gstart[g] .. gstart[g+1])
  const uint64_t* Es;
  const int64_t* yq;
  const double* y;
  const double* X;
  int64_t ldx;
  int64_t n;
  int p, mtry, nodesize, q, A;
  uint64_t seed;
  int32_t t0;
  Pool pool;
  unsigned long long* stats;  // optional phase counters (BF_SUBTREE_STATS=1), else NULL
  unsigned long long* visits; // optional (profile mode): split-search entry visits (mtry x distinct rows per node)
  int tq_sleep_max;           // idle-warp back-off cap in ns (BF_TQ_SLEEP_MAX, default 512)
  int tq_bigger_first;        // continue with the child of more distinct rows (BF_TQ_BIGGER_FIRST, default 1)
  int tq_lpt;                 // tiny roots queued before the tiny phase taken largest first (BF_TQ_LPT, default 1)
};

// S4.2 mtry draw by one warp, in parallel.  Draw i picks position
// j_i = mulhi64(U_i, p - i) of the current array, then swaps positions j_i
// and p-1-i.  The content of position x after draws 0..i-1 is found by
// tracing the swaps backwards (x <- p-1-k if x == j_k, x <- j_k if
// x == p-1-k, for k = i-1 .. 0), so lane i computes feature i on its own
// from the j values of the earlier draws (kept in shared memory).
__device__ __forceinline__ void warp_draw_mtry(uint64_t seed, uint32_t t, uint64_t key, int p, int mtry, int16_t* jbuf,
                                               int16_t* feats, int lane) {
  if (mtry <= 32) {  // one draw per lane; the earlier draws' j come by shuffle (no shared-memory round trips)
    int j = 0;
    if (lane < mtry) {
      uint64_t u0, u1;
      philox_u64x2(seed, (uint32_t)key, (uint32_t)(key >> 32), t, 0x20000000u | (uint32_t)(lane >> 1), u0, u1);
      j = (int)mulhi64((lane & 1) ? u1 : u0, (uint64_t)(p - lane));
    }
    int x = j;
#pragma unroll 4
    for (int k = mtry - 2; k >= 0; --k) {  // lane i applies k = i-1 .. 0 (warp-uniform loop)
      const int jk = __shfl_sync(0xffffffffu, j, k), lk = p - 1 - k;
      if (k < lane) x = (x == jk) ? lk : ((x == lk) ? jk : x);
    }
    if (lane < mtry) feats[lane] = (int16_t)x;
    __syncwarp();
    return;
  }
  for (int i0 = 0; i0 < mtry; i0 += 32) {
    const int i = i0 + lane;
    if (i < mtry) {
      uint64_t u0, u1;
      philox_u64x2(seed, (uint32_t)key, (uint32_t)(key >> 32), t, 0x20000000u | (uint32_t)(i >> 1), u0, u1);
      jbuf[i] = (int16_t)mulhi64((i & 1) ? u1 : u0, (uint64_t)(p - i));
    }
  }
  __syncwarp();
  for (int i0 = 0; i0 < mtry; i0 += 32) {
    const int i = i0 + lane;
    if (i < mtry) {
      int x = jbuf[i];
#pragma unroll 4
      for (int k = i - 1; k >= 0; --k) {
        const int jk = jbuf[k], lk = p - 1 - k;
        x = (x == jk) ? lk : ((x == lk) ? jk : x);
      }
      feats[i] = (int16_t)x;
    }
  }
  __syncwarp();
}

// Tiny-node work queue (shared memory).  Every access to a queue entry, its ready flag and the queue
// counters is an atomic read-modify-write through cuda::atomic_ref (block scope): the producer writes the
// entry's fields with relaxed exchanges and publishes it with a release exchange of ready[idx]; the consumer's
// lane 0 spins on an acquire fetch_or(0) of the flag, reads the fields with relaxed fetch_or(0) and broadcasts
// them to its warp.  The hand-off is ordered by the memory model (release/acquire on the flag), and since
// every cross-warp access is an atomic RMW, compute-sanitizer's racecheck (which models barriers and atomics,
// not ld/st.acquire/release) has no plain shared-memory access to report.
template <class T>
using blk_ref = cuda::atomic_ref<T, cuda::thread_scope_block>;
using u64 = unsigned long long;

template <class T>
__device__ __forceinline__ void a_put(T& x, T v) {
  blk_ref<T>(x).exchange(v, cuda::memory_order_relaxed);
}
template <class T>
__device__ __forceinline__ T a_get(T& x) {
  return blk_ref<T>(x).fetch_or(T(0), cuda::memory_order_relaxed);
}

template <int NWD>
__device__ __forceinline__ void tq_push(TNodeT<NWD>* q, int32_t* ready, int* alloc, int* pending,
                                        const TNodeT<NWD>& c) {
  atomicAdd(pending, 1);
  const int idx = atomicAdd(alloc, 1);
  TNodeT<NWD>& e = q[idx];
  a_put<int32_t>(e.rlo, c.rlo);
  a_put<int32_t>(e.ra, c.ra);
#pragma unroll
  for (int w = 0; w < NWD; ++w) a_put<u64>(*(u64*)&e.mask[w], (u64)c.mask[w]);
  a_put<int32_t>(e.id, c.id);
  a_put<int32_t>(e.n, c.n);
  a_put<u64>(*(u64*)&e.S, (u64)c.S);
  a_put<u64>(*(u64*)&e.key, (u64)c.key);
  a_put<u64>(*(u64*)&e.value, (u64)__double_as_longlong(c.value));
  blk_ref<int32_t>(ready[idx]).exchange(1, cuda::memory_order_release);
}

template <int NWD>
__device__ __forceinline__ TNodeT<NWD> tq_read(TNodeT<NWD>* q, int idx) {  // after an acquire of ready[idx] (or a barrier)
  TNodeT<NWD>& e = q[idx];
  TNodeT<NWD> c;
  c.rlo = a_get<int32_t>(e.rlo);
  c.ra = a_get<int32_t>(e.ra);
#pragma unroll
  for (int w = 0; w < NWD; ++w) c.mask[w] = (uint64_t)a_get<u64>(*(u64*)&e.mask[w]);
  c.id = a_get<int32_t>(e.id);
  c.n = a_get<int32_t>(e.n);
  c.S = (int64_t)a_get<u64>(*(u64*)&e.S);
  c.key = (uint64_t)a_get<u64>(*(u64*)&e.key);
  c.value = __longlong_as_double((long long)a_get<u64>(*(u64*)&e.value));
  return c;
}

template <int NWD>
__device__ __forceinline__ TNodeT<NWD> tq_bcast(const TNodeT<NWD>& c) {  // lane 0's entry to the whole warp
  TNodeT<NWD> r;
  r.rlo = __shfl_sync(0xffffffffu, c.rlo, 0);
  r.ra = __shfl_sync(0xffffffffu, c.ra, 0);
#pragma unroll
  for (int w = 0; w < NWD; ++w) r.mask[w] = __shfl_sync(0xffffffffu, c.mask[w], 0);
  r.id = __shfl_sync(0xffffffffu, c.id, 0);
  r.n = __shfl_sync(0xffffffffu, c.n, 0);
  r.S = __shfl_sync(0xffffffffu, c.S, 0);
  r.key = __shfl_sync(0xffffffffu, c.key, 0);
  r.value = __shfl_sync(0xffffffffu, c.value, 0);
  return r;
}

// TV: tiny-node search (0 staged warp items, 1 lane per drawn feature with a position table, 2 lane per drawn
// feature with ballot masks); TT: largest tiny root (64 or 128 rows); HW: helper warps that grow tiny nodes
// while the other SUB_NW - HW warps run the medium levels (named barrier 1), 0 = phases in sequence
template <int TV, int TT, int HW>
__global__ void __launch_bounds__(SUB_NT) k_subtree(SubArgs g) {
  static_assert(TT == 64 || (TT == 128 && (TV == 1 || TV == 3)), "tiny roots of 128 rows need the position table");
  static_assert(HW == 0 || TV == 2, "helper warps need the ballot masks (no position table during the medium levels)");
  constexpr int NMW = SUB_NW - HW;  // warps of the medium levels
  auto mbar = [&]() {
    if constexpr (HW == 0) __syncthreads();
    else asm volatile("bar.sync 1, %0;" ::"r"(NMW * 32) : "memory");
  };
  constexpr bool LPF = TV >= 1;  // lane-per-feature tiny search (1: masks from the position table, 2: by ballots,
                                 // 3: position table built per tiny root by the warp that takes the root)
  constexpr int ROOTF = 1 << 30;  // TV 3: queue entry of a tiny root whose rmap / ppos are not built yet (in ra)
  constexpr int NWD = TT / 64;
  using TN = TNodeT<NWD>;
  extern __shared__ __align__(16) unsigned char smem[];
  const int A = g.A, p = g.p, MM = max_medium(A);
  unsigned char* ptr = smem;
  uint32_t* list = (uint32_t*)ptr;
  ptr += align16((size_t)p * A * 4);
  uint32_t* temp_all = (uint32_t*)ptr;
  ptr += align16(sub_temp_bytes(A, p));
  int64_t* wy = (int64_t*)ptr;
  ptr += align16((size_t)A * 8);
  double* wyd = (double*)ptr;
  ptr += align16((size_t)A * 8);
  int32_t* wl = (int32_t*)ptr;
  ptr += align16((size_t)A * 4);
  uint32_t* grow = (uint32_t*)ptr;
  ptr += align16((size_t)A * 4);
  uint8_t* side = (uint8_t*)ptr;
  ptr += align16((size_t)A);
  uint8_t* rmap = (uint8_t*)ptr;
  ptr += align16((size_t)A);
  SRec* recs = (SRec*)ptr;
  ptr += align16((size_t)2 * A * sizeof(SRec));
  // DEFER (lane-per-feature search, 64-row tiny roots): the value of a tiny-phase record is computed at the flush
  // from its row mask (held in the record's value field) over its tiny root's rows, off the critical path
  constexpr bool DEFER = LPF && NWD == 1;
  uint16_t* rdef = (uint16_t*)ptr;
  ptr += align16((size_t)2 * A * 2);
  MNode* curl = (MNode*)ptr;
  MNode* nxtl = curl + MM;
  ptr += align16((size_t)2 * MM * sizeof(MNode));
  TN* tq = (TN*)ptr;
  ptr += align16((size_t)(A + MAXR) * sizeof(TN));
  int32_t* tq_ready = (int32_t*)ptr;
  ptr += align16((size_t)(A + MAXR) * 4);
  int16_t* mind_all = (int16_t*)ptr;
  ptr += align16((size_t)SUB_NW * p * 2);
  int16_t* feats_all = (int16_t*)ptr;
  ptr += align16((size_t)SUB_NW * p * 2);
  WRec* wrec = (WRec*)ptr;
  ptr += align16((size_t)SUB_NW * sizeof(WRec));
  __shared__ int s_ncur, s_alloc, s_head, s_pending;
  __shared__ int32_t s_scan[SUB_NW];
  // packed roots: local rows [s_off[r], s_off[r+1]), records [2 s_off[r], ...) (a tree over a rows has < 2a
  // nodes), next free record s_nloc[r]; node ids carry their root: id = r << 16 | record
  __shared__ int s_off[MAXR + 1], s_b[MAXR], s_nloc[MAXR], s_gbase[MAXR];
  __shared__ LNode s_root[MAXR];

  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int g0 = g.gstart[blockIdx.x], nr = g.gstart[blockIdx.x + 1] - g0;
  if (tid < nr) s_root[tid] = g.sq[g.gperm[g0 + tid]];
  __syncthreads();
  if (tid == 0) {
    int o = 0;
    for (int r = 0; r < nr; ++r) {
      s_off[r] = o;
      s_b[r] = s_root[r].b;
      s_nloc[r] = 2 * o + 1;
      o += s_root[r].a;
    }
    s_off[nr] = o;
  }
  __syncthreads();
  const int a0 = s_off[nr];  // rows of all packed roots = the stride of a feature row of `list`
  auto t_of = [&](int32_t id) -> uint32_t { return (uint32_t)(g.t0 + s_b[id >> 16]); };
  auto root_of_row = [&](int j) -> int {  // packed root holding local row j
    int r = 0;
    while (r + 1 < nr && s_off[r + 1] <= j) ++r;
    return r;
  };
  int16_t* mind = mind_all + wid * p;
  int16_t* feats = feats_all + wid * p;
  uint32_t* temp = temp_all + (size_t)wid * sub_temp(A);
  long long tclk[5];
  tclk[0] = clock64();
  int n_med = 0, n_tiny = 0;
  long long busy = 0;
  unsigned long long nvis = 0;  // entry visits of this warp's split searches (profile mode)

  // ---- load 1: local rows = feature 0's order; payload; global row -> local id in a shared-memory hash
  // table (open addressing over HSLOTS slots, built in the scratch area that the later phases reuse)
  uint32_t* hkey = temp_all;
  uint16_t* hval = (uint16_t*)(temp_all + HSLOTS);
  for (int k = tid; k < HSLOTS; k += SUB_NT) hkey[k] = 0xffffffffu;
  __syncthreads();
  for (int j = tid; j < a0; j += SUB_NT) {
    const int r = root_of_row(j);
    const uint64_t ej = g.Es[s_root[r].base + (j - s_off[r])];  // feature 0's segment of root r
    const uint32_t row = e_row(ej);
    const int32_t wv = e_w(ej);
    const int64_t yqr = g.yq[row];
    const double yr = g.y[row];
    grow[j] = row;
    const uint32_t hk = row | ((uint32_t)r << 24);  // the same row may sit in two packed roots (two trees)
    uint32_t h = (hk * 0x9E3779B1u) >> (32 - HBITS);
    while (atomicCAS(&hkey[h], 0xffffffffu, hk) != 0xffffffffu) h = (h + 1) & (HSLOTS - 1);
    hval[h] = (uint16_t)j;
    wl[j] = wv;
    wy[j] = (int64_t)wv * yqr;
    wyd[j] = __dmul_rn((double)wv, yr);
  }
  for (int j = tid; j < a0 + MAXR; j += SUB_NT) tq_ready[j] = 0;  // barrier-ordered before any queue use
  for (int j = tid; j < 2 * a0; j += SUB_NT) rdef[j] = 0xffffu;
  __syncthreads();
  auto hfind = [&](uint32_t hk) -> uint16_t {
    uint32_t h = (hk * 0x9E3779B1u) >> (32 - HBITS);
    while (hkey[h] != hk) h = (h + 1) & (HSLOTS - 1);
    return hval[h];
  };
  // ---- load 2: warp per feature; local rank = index of the first entry of the same value.  Coalesced: chunk c
  // of 32 entries is read by lane l at entry 32c + l, each entry once (rank and row from the same 8-byte load),
  // up to 16 chunks (a0 <= 512) in flight per warp; the value breaks are max-scanned per chunk with a carry.
  {
    constexpr int GRP = 16;
    for (int it = wid; it < nr * p; it += SUB_NW) {  // (packed root, feature) items
      const int r = it / p, f = it - r * p;
      const int ar = s_root[r].a, orr = s_off[r];
      const int nch = (ar + 31) >> 5;
      const uint64_t* sf = g.Es + s_root[r].base + (int64_t)f * ar;
      const uint32_t rtag = (uint32_t)r << 24;
      int carry_gs = 0;
      uint32_t prev_last = 0xffffffffu;
      for (int c0 = 0; c0 < nch; c0 += GRP) {
        uint64_t ev[GRP];
#pragma unroll
        for (int c = 0; c < GRP; ++c) {
          const int j = (c0 + c) * 32 + lane;
          ev[c] = (c0 + c < nch && j < ar) ? sf[j] : ~0ull;
        }
        uint32_t rk[GRP];
        uint16_t lr[GRP];
#pragma unroll
        for (int c = 0; c < GRP; ++c) {
          const int j = (c0 + c) * 32 + lane;
          rk[c] = j < ar ? e_rank(ev[c]) : 0xffffffffu;
          lr[c] = (c0 + c < nch && j < ar) ? hfind(e_row(ev[c]) | rtag) : 0;
        }
#pragma unroll
        for (int c = 0; c < GRP; ++c) {
          if (c0 + c >= nch) break;
          const int j = (c0 + c) * 32 + lane;
          const uint32_t up = __shfl_up_sync(0xffffffffu, rk[c], 1);
          const uint32_t prv = lane == 0 ? prev_last : up;
          int gs = (j > 0 && rk[c] != prv) ? j : 0;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const int v = __shfl_up_sync(0xffffffffu, gs, o);
            if (lane >= o) gs = max(gs, v);
          }
          gs = max(gs, carry_gs);
          if (j < ar) list[(size_t)f * a0 + orr + j] = ((uint32_t)(orr + gs) << 16) | lr[c];
          carry_gs = __shfl_sync(0xffffffffu, gs, 31);
          prev_last = __shfl_sync(0xffffffffu, rk[c], 31);
        }
      }
    }
  }
  if (tid == 0) {
    s_head = 0;
    s_alloc = 0;
    s_pending = 0;
    s_ncur = 0;
  }
  __syncthreads();
  if (tid < nr) {  // each packed root: its record, then a medium node or a tiny root
    const int r = tid;
    const LNode& R = s_root[r];
    const int rec0 = 2 * s_off[r];
    SRec r0;
    r0.feature = -1;
    r0.left = -1;
    r0.count = R.n;
    r0.ra = r0.rb = 0;
    r0.value = 0.0;
    r0.drss = 0.0;
    recs[rec0] = r0;
    if (R.a > TT) {
      MNode c;
      c.lo = s_off[r];
      c.a = R.a;
      c.n = R.n;
      c.id = (r << 16) | rec0;
      c.S = R.S;
      c.key = R.key;
      c.split = 0;
      curl[atomicAdd(&s_ncur, 1)] = c;
    } else {
      TN c;
      c.rlo = s_off[r];
      c.ra = R.a;
      m_full(c.mask, R.a);
      if constexpr (TV == 3) c.ra |= ROOTF;
      c.id = (r << 16) | rec0;
      c.n = R.n;
      c.S = R.S;
      c.key = R.key;
      c.value = 0.0;  // a root's value is the pool's (written before the subtree phase)
      if constexpr (HW > 0)  // row index inside the tiny root, before it is published
        for (int k = 0; k < R.a; ++k) rmap[list[s_off[r] + k] & 0xffffu] = (uint8_t)k;
      tq_push(tq, tq_ready, &s_alloc, &s_pending, c);
    }
  }
  __shared__ int s_mdone, s_nidx[16];
  if (tid == 0) s_mdone = 0;
  __syncthreads();
  tclk[1] = clock64();

  // ================= medium levels (a > TINY): level-synchronous inside the CTA
  long long mclk[3] = {0, 0, 0};  // medium phase: scan+finalize, next level, partition (thread 0, stats only)
  long long mfin = 0;             // of which finalize (warp per node after the item barrier)
  int n_mlev = 0;                 // medium levels
  if (HW == 0 || wid < NMW) {
  while (s_ncur > 0) {
    const long long mc0 = clock64();
    const int ncur = s_ncur;
    n_med += ncur;
    ++n_mlev;
    // (node, drawn predictor) items over all warps; per-item winners in the scratch area; one warp per node
    // reduces its items (lowest predictor on equal keys) and finalizes the split.  Nodes go in groups whose
    // items fit the scratch area (and whose draws fit the per-warp feature slots).
    WRec* irec = (WRec*)temp_all;  // the medium warps' scratch (helper warps keep theirs)
    const int cap_items = (int)((size_t)NMW * sub_temp(A) * 4 / sizeof(WRec));
    const int NG = max(1, min(NMW, cap_items / g.mtry));
    for (int n0 = 0; n0 < ncur; n0 += NG) {
      const int nn = min(NG, ncur - n0);
      if (wid < nn) warp_draw_mtry(g.seed, t_of(curl[n0 + wid].id), curl[n0 + wid].key, p, g.mtry, mind_all + wid * p, feats_all + wid * p, lane);
      mbar();
      const int nit = nn * g.mtry;
      for (int it = wid; it < nit; it += NMW) {
        const int li = it / g.mtry;
        const MNode nd = curl[n0 + li];
        const int f = feats_all[li * p + (it - li * g.mtry)];
        const uint32_t* seg = list + (size_t)f * a0 + nd.lo;
        const int64_t nk = nd.n, Sk = nd.S;
        const float nkf = __ll2float_rn(nk), Skf = __ll2float_rn(Sk);
          double lg = -1.0;
        uint32_t lrk = 0xffffffffu, lra = 0, lrb = 0;
        int lpos = -1, lnl = 0;
        int64_t lSl = 0;
        // K consecutive entries per lane: lane-serial sums, one warp scan, a bounds pass screened by the
        // warp max of the lower bounds (and the warp's best so far), exact keys only where they may win
        const int aN = nd.a, K = (aN + 31) >> 5;
        nvis += (unsigned)aN;
        const int i0 = min(lane * K, aN), i1 = min(i0 + K, aN);
        int32_t rw = 0;
        int64_t rsum = 0;
#pragma unroll 4
        for (int i = i0; i < i1; ++i) {
          const uint32_t lr = seg[i] & 0xffffu;
          rw += wl[lr];
          rsum += wy[lr];
        }
        const int32_t cw0 = warp_incl_scan(rw, lane) - rw;
        const int64_t cs0 = warp_incl_scan(rsum, lane) - rsum;
        float mL = -1.0f, mU = -1.0f, u2 = -1.0f;  // fp32 t-space screen; largest / second largest upper bound
        int bi = -1;
        int32_t bcw = 0;
        int64_t bcs = 0;
        {
          int32_t cw = cw0;
          int64_t cs = cs0;
#pragma unroll 2
          for (int i = i0; i < i1; ++i) {
            const uint32_t e = seg[i], lr = e & 0xffffu;
            cw += wl[lr];
            cs += wy[lr];
            if (i + 1 < aN && (seg[i + 1] >> 16) != (e >> 16)) {
              float gL, gU;
              key_bounds_t(nkf, Skf, nk, cw, cs, gL, gU);
              mL = fmaxf(mL, gL);
              if (gU > mU) {
                u2 = mU;
                mU = gU;
                bi = i;
                bcw = cw;
                bcs = cs;
              } else {
                u2 = fmaxf(u2, gU);
              }
            }
          }
        }
        const float M = warp_max_t(mL);
        if (mU >= M && mU >= 0.0f && u2 < M) {  // a single candidate item on this lane
          const uint32_t e = seg[bi], en = seg[bi + 1];
          const double gk = split_key(nk, Sk, bcw, bcs);
          if (rec_better(gk, e >> 16, lg, lrk)) {
            lg = gk;
            lrk = e >> 16;
            lra = e & 0xffffu;
            lrb = en & 0xffffu;
            lpos = bi;
            lnl = bcw;
            lSl = bcs;
          }
        } else if (mU >= M && mU >= 0.0f) {
          int32_t cw = cw0;
          int64_t cs = cs0;
          for (int i = i0; i < i1; ++i) {
            const uint32_t e = seg[i], lr = e & 0xffffu;
            cw += wl[lr];
            cs += wy[lr];
            if (i + 1 < aN) {
              const uint32_t en = seg[i + 1];
              if ((en >> 16) != (e >> 16)) {
                float gL, gU;
                key_bounds_t(nkf, Skf, nk, cw, cs, gL, gU);
                if (gU >= M) {
                  const double gk = split_key(nk, Sk, cw, cs);
                  if (rec_better(gk, e >> 16, lg, lrk)) {
                    lg = gk;
                    lrk = e >> 16;
                    lra = lr;
                    lrb = en & 0xffffu;
                    lpos = i;
                    lnl = cw;
                    lSl = cs;
                  }
                }
              }
            }
          }
        }
        const int srcl = max(warp_argmax_key(gkey(lg), lrk), 0);
        lg = __shfl_sync(0xffffffffu, lg, srcl);
        lrk = __shfl_sync(0xffffffffu, lrk, srcl);
        const int wpos = __shfl_sync(0xffffffffu, lpos, srcl);
        const int wnl = __shfl_sync(0xffffffffu, lnl, srcl);
        const int64_t wSl = __shfl_sync(0xffffffffu, lSl, srcl);
        const uint32_t wra = __shfl_sync(0xffffffffu, lra, srcl);
        const uint32_t wrb = __shfl_sync(0xffffffffu, lrb, srcl);
        if (lane == 0) {
          WRec r;
          r.g = lg >= 0.0 ? lg : -1.0;
          r.f = f;
          r.lrank = lrk;
          r.pos = wpos;
          r.nl = wnl;
          r.Sl = wSl;
          r.ra = wra;
          r.rb = wrb;
          irec[it] = r;
        }
      }
      mbar();
      const long long mf0 = clock64();
      if (wid < nn) {
        const int i = n0 + wid;
        MNode nd = curl[i];
        // the node's best item: lane-local over its items, then the warp (key desc, predictor asc)
        double lgb = -1.0;
        int lfb = 0x7fffffff, lsb = -1;
        for (int s2 = lane; s2 < g.mtry; s2 += 32) {
          const WRec& r = irec[wid * g.mtry + s2];
          if (r.g >= 0.0 && (r.g > lgb || (r.g == lgb && r.f < lfb))) {
            lgb = r.g;
            lfb = r.f;
            lsb = s2;
          }
        }
        const int wln = warp_argmax_key(gkey(lgb), (uint32_t)lfb);
        const int sb = __shfl_sync(0xffffffffu, lsb, wln >= 0 ? wln : 0);
        WRec best;
        best.g = -1.0;
        if (wln >= 0) best = irec[wid * g.mtry + sb];
        if (best.g > 0.0) {
          int lid = 0;
          if (lane == 0) {
            lid = atomicAdd(&s_nloc[nd.id >> 16], 2);
            SRec& r = recs[nd.id & 0xffff];
            r.feature = best.f;
            r.left = lid;
            r.ra = (uint16_t)best.ra;
            r.rb = (uint16_t)best.rb;
            r.drss = ldexp(__ddiv_rn(best.g, (double)nd.n), -2 * g.q);
            nd.keyl = child_key(g.seed, t_of(nd.id), nd.key, 0);
            nd.keyr = child_key(g.seed, t_of(nd.id), nd.key, 1);
          }
          lid = __shfl_sync(0xffffffffu, lid, 0);
          const uint32_t* seg = list + (size_t)best.f * a0 + nd.lo;
          double sl = 0.0, sr = 0.0;
          for (int j = lane; j < nd.a; j += 32) {
            const uint32_t lr = seg[j] & 0xffffu;
            const int sdv = j > best.pos;
            side[lr] = (uint8_t)sdv;
            if (sdv) sr += wyd[lr];
            else sl += wyd[lr];
          }
#pragma unroll
          for (int o = 16; o > 0; o >>= 1) {
            sl += __shfl_down_sync(0xffffffffu, sl, o);
            sr += __shfl_down_sync(0xffffffffu, sr, o);
          }
          if (lane == 0) {
            const int nr = nd.n - best.nl, al = best.pos + 1, ar = nd.a - al;
            SRec c;
            c.feature = -1;
            c.left = -1;
            c.ra = c.rb = 0;
            c.drss = 0.0;
            c.count = best.nl;
            c.value = __ddiv_rn(sl, (double)best.nl);
            recs[lid] = c;
            c.count = nr;
            c.value = __ddiv_rn(sr, (double)nr);
            recs[lid + 1] = c;
            nd.split = 1;
            nd.lid = lid;
            nd.al = al;
            nd.nl = best.nl;
            nd.Sl = best.Sl;
            nd.kind[0] = (best.nl <= g.nodesize || al < 2) ? KIND_LEAF : (al <= TT ? KIND_SMALL : KIND_LARGE);
            nd.kind[1] = (nr <= g.nodesize || ar < 2) ? KIND_LEAF : (ar <= TT ? KIND_SMALL : KIND_LARGE);
            curl[i] = nd;
          }
        } else if (lane == 0) {
          curl[i].split = 0;
        }
      }
      mbar();
      mfin += clock64() - mf0;
    }
    const long long mc1 = clock64();
    // ---- next medium level (block scan) and tiny roots (work queue; processed after the medium levels, or by
    // the helper warps once the level's partition is done)
    {
      int kc = 0;
      MNode nd;
      if (tid < ncur) {
        nd = curl[tid];
        if (nd.split) kc = (nd.kind[0] == KIND_LARGE) + (nd.kind[1] == KIND_LARGE);
      }
      int totc, idx;
      if constexpr (HW == 0) {
        idx = block_excl_scan(kc, s_scan, totc);
      } else {  // ncur <= max_medium(A) nodes: one thread's running sum
        if (tid < ncur) s_nidx[tid] = kc;
        mbar();
        if (tid == 0) {
          int run = 0;
          for (int i = 0; i < ncur; ++i) {
            const int v = s_nidx[i];
            s_nidx[i] = run;
            run += v;
          }
          s_ncur = run;
        }
        mbar();
        idx = tid < ncur ? s_nidx[tid] : 0;
        totc = 0;
      }
      if (tid < ncur && nd.split) {
        for (int sdv = 0; sdv < 2; ++sdv) {
          const int kd = nd.kind[sdv];
          if (kd == KIND_LEAF) continue;
          const int lo = sdv ? nd.lo + nd.al : nd.lo;
          const int a = sdv ? nd.a - nd.al : nd.al;
          const int nn = sdv ? nd.n - nd.nl : nd.nl;
          const int64_t S = sdv ? nd.S - nd.Sl : nd.Sl;
          const uint64_t key = sdv ? nd.keyr : nd.keyl;
          if (kd == KIND_LARGE) {
            MNode c;
            c.lo = lo;
            c.a = a;
            c.n = nn;
            c.id = (nd.id & ~0xffff) | (nd.lid + sdv);
            c.S = S;
            c.key = key;
            c.split = 0;
            nxtl[idx++] = c;
          } else {
            TN c;
            c.rlo = lo;
            c.ra = a;
            m_full(c.mask, a);
            if constexpr (TV == 3) c.ra |= ROOTF;
            c.id = (nd.id & ~0xffff) | (nd.lid + sdv);
            c.n = nn;
            c.S = S;
            c.key = key;
            c.value = recs[nd.lid + sdv].value;  // written by the node's warp before the last barrier
            if constexpr (HW == 0) tq_push(tq, tq_ready, &s_alloc, &s_pending, c);
          }
        }
      }
      if (HW == 0 && tid == 0) s_ncur = totc;
    }
    const long long mc2 = clock64();
    // ---- in-place stable partition of every feature row of every split node with a non-leaf child
    for (int it = wid; it < ncur * p; it += NMW) {
      const int i = it / p, f = it - i * p;
      const MNode& nd = curl[i];
      if (!nd.split || (nd.kind[0] == KIND_LEAF && nd.kind[1] == KIND_LEAF)) continue;
      uint32_t* seg = list + (size_t)f * a0 + nd.lo;
      const int al = nd.al;
      const int aN = nd.a;
      int carry = 0;
      for (int j0 = 0; j0 < aN; j0 += 128) {  // 4 rows of 32 with their loads in flight together
        uint32_t e[4];
        int sdv[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) e[u] = j0 + 32 * u + lane < aN ? seg[j0 + 32 * u + lane] : 0u;
#pragma unroll
        for (int u = 0; u < 4; ++u) sdv[u] = j0 + 32 * u + lane < aN ? side[e[u] & 0xffffu] : 1;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int j = j0 + 32 * u + lane;
          const bool valid = j < aN;
          const unsigned m = __ballot_sync(0xffffffffu, valid && sdv[u] == 0);
          const int lb = carry + __popc(m & ((1u << lane) - 1u));
          if (valid) temp[sdv[u] ? al + (j - lb) : lb] = e[u];
          carry += __popc(m);
        }
      }
      __syncwarp();
      for (int j0 = 0; j0 < aN; j0 += 128) {
        uint32_t v[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) v[u] = j0 + 32 * u + lane < aN ? temp[j0 + 32 * u + lane] : 0u;
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (j0 + 32 * u + lane < aN) seg[j0 + 32 * u + lane] = v[u];
      }
      __syncwarp();
    }
    mbar();
    if constexpr (HW > 0) {  // the level's tiny children: lists final now; row index, then publish (warp per node)
      for (int i = wid; i < ncur; i += NMW) {
        const MNode nd = curl[i];
        if (!nd.split) continue;
        for (int sdv = 0; sdv < 2; ++sdv) {
          if (nd.kind[sdv] != KIND_SMALL) continue;
          TN c;
          c.rlo = sdv ? nd.lo + nd.al : nd.lo;
          c.ra = sdv ? nd.a - nd.al : nd.al;
          m_full(c.mask, c.ra);
          c.id = (nd.id & ~0xffff) | (nd.lid + sdv);
          c.n = sdv ? nd.n - nd.nl : nd.nl;
          c.S = sdv ? nd.S - nd.Sl : nd.Sl;
          c.key = sdv ? nd.keyr : nd.keyl;
          c.value = recs[nd.lid + sdv].value;
          for (int k = lane; k < c.ra; k += 32) rmap[list[c.rlo + k] & 0xffffu] = (uint8_t)k;
          __syncwarp();
          if (lane == 0) tq_push(tq, tq_ready, &s_alloc, &s_pending, c);
        }
      }
    }
    {
      const long long mc3 = clock64();
      mclk[0] += mc1 - mc0;
      mclk[1] += mc2 - mc1;
      mclk[2] += mc3 - mc2;
      MNode* tl = curl;
      curl = nxtl;
      nxtl = tl;
    }
  }
  if constexpr (HW > 0) {
    mbar();  // every medium warp has published its tiny roots
    if (tid == 0) blk_ref<int>(s_mdone).exchange(1, cuda::memory_order_release);
  }
  }  // medium warps

  // ================= tiny nodes: row index inside each tiny root, then the work queue
  tclk[2] = clock64();
  if constexpr (HW == 0 && TV != 3) {
    const int nroots = a_get<int>(s_alloc);
    for (int qi = wid; qi < nroots; qi += SUB_NW) {
      const TN r = tq_read(tq, qi);  // pushed before the barrier above
      for (int k = lane; k < r.ra; k += 32) rmap[list[r.rlo + k] & 0xffffu] = (uint8_t)k;
    }
    __syncthreads();
  }
  // TV = 1: ppos[f * a0 + rlo + i] = position, in feature f's segment of its tiny root, of the row at feature-0
  // position i (the scratch area is free once the medium levels are done), so a node's rows in feature f's order
  // are the set bits of one 64-bit mask built from the node's mask (no staging, no pass over non-member rows)
  uint8_t* ppos = (uint8_t*)temp_all;
  if constexpr (TV == 1) {  // (TV 2 builds its masks by ballots instead)
    const int nroots = a_get<int>(s_alloc);
    for (int it = wid; it < nroots * p; it += SUB_NW) {
      const int qi = it / p, f = it - qi * p;
      const int rlo = a_get<int32_t>(tq[qi].rlo), ra = a_get<int32_t>(tq[qi].ra);
      const uint32_t* seg = list + (size_t)f * a0 + rlo;
      uint8_t* pp = ppos + (size_t)f * a0 + rlo;
      for (int k = lane; k < ra; k += 32) pp[rmap[seg[k] & 0xffffu]] = (uint8_t)k;
    }
    __syncthreads();
  }
  // The tiny roots queued before this phase are taken largest first (longest-processing-time order: the longest
  // chains start first, so the tail of the phase is shorter).  rorder[h] = queue entry of the h-th pop, in the
  // `side` bytes (free after the medium levels); up to 64 roots (else queue order).
  int16_t* rorder = reinterpret_cast<int16_t*>(side);
  __shared__ int s_nr0;
  if (HW == 0 && wid == 0) {
    const int nr0 = a_get<int>(s_alloc);
    const bool lpt = g.tq_lpt && nr0 <= 64 && 2 * nr0 <= A;
    if (lpt) {
      const int i0 = lane, i1 = lane + 32;
      const int k0 = i0 < nr0 ? a_get<int32_t>(tq[i0].ra) : -1, k1 = i1 < nr0 ? a_get<int32_t>(tq[i1].ra) : -1;
      int r0 = 0, r1 = 0;
      for (int j = 0; j < nr0; ++j) {
        const int kj = __shfl_sync(0xffffffffu, j < 32 ? k0 : k1, j & 31);
        r0 += (kj > k0) || (kj == k0 && j < i0);
        r1 += (kj > k1) || (kj == k1 && j < i1);
      }
      if (i0 < nr0) rorder[r0] = (int16_t)i0;
      if (i1 < nr0) rorder[r1] = (int16_t)i1;
    }
    if (lane == 0) s_nr0 = lpt ? nr0 : 0;
  }
  if constexpr (HW == 0) __syncthreads();
  const int nr0 = HW == 0 ? s_nr0 : 0;
  for (;;) {
    int h = -1;
    TN nd;
    if (lane == 0) {
      unsigned ns = 32;
      for (;;) {
        const int hd = a_get<int>(s_head);
        if (hd < a_get<int>(s_alloc)) {
          if (atomicCAS(&s_head, hd, hd + 1) == hd) {
            h = hd;
            break;
          }
        } else if (a_get<int>(s_pending) == 0 && (HW == 0 || a_get<int>(s_mdone) != 0)) {
          break;
        } else {
          __nanosleep(ns);  // idle warp: back off so the busy warps keep the issue slots
          ns = min(ns * 2, (unsigned)g.tq_sleep_max);
        }
      }
      if (h >= 0) {
        if (h < nr0) h = rorder[h];  // a root queued before the phase: largest first
        while (blk_ref<int32_t>(tq_ready[h]).fetch_or(0, cuda::memory_order_acquire) == 0) __nanosleep(32);
        nd = tq_read(tq, h);
      }
    }
    h = __shfl_sync(0xffffffffu, h, 0);
    if (h < 0) break;
    nd = tq_bcast(nd);
    bool have = true;
    const long long tb0 = clock64();
    while (have) {
      have = false;
      ++n_tiny;
      if constexpr (TV == 3) {
        if (nd.ra & ROOTF) {  // first node of a tiny root: its row index and position table, by this warp
          nd.ra &= ~ROOTF;
          const int rl = nd.rlo, rr = nd.ra;
          for (int k = lane; k < rr; k += 32) rmap[list[rl + k] & 0xffffu] = (uint8_t)k;
          __syncwarp();
          constexpr int FU = 16 / (TT / 32);  // features per round: 16 loads in flight per lane
          for (int f0 = 0; f0 < p; f0 += FU) {
            uint32_t ev[FU * (TT / 32)];
#pragma unroll
            for (int u = 0; u < FU; ++u) {
              const uint32_t* sg = list + (size_t)min(f0 + u, p - 1) * a0 + rl;
#pragma unroll
              for (int hh = 0; hh < TT / 32; ++hh) ev[u * (TT / 32) + hh] = lane + 32 * hh < rr ? sg[lane + 32 * hh] : 0u;
            }
#pragma unroll
            for (int u = 0; u < FU; ++u) {
              uint8_t* pp = ppos + (size_t)min(f0 + u, p - 1) * a0 + rl;
#pragma unroll
              for (int hh = 0; hh < TT / 32; ++hh)
                if (f0 + u < p && lane + 32 * hh < rr)
                  pp[rmap[ev[u * (TT / 32) + hh] & 0xffffu]] = (uint8_t)(lane + 32 * hh);
            }
          }
          __syncwarp();
        }
      }
      const int rlo = nd.rlo, ra = nd.ra;
      const int an = m_popc(nd.mask);  // distinct rows of the node
      nvis += (unsigned long long)an * (unsigned)g.mtry;
      const long long c0_ = g.stats ? clock64() : 0;
      const uint32_t t = t_of(nd.id);
      warp_draw_mtry(g.seed, t, nd.key, p, g.mtry, mind, feats, lane);
      const uint64_t ck = child_key(g.seed, t, nd.key, lane & 1);  // independent of the split: off the tail
      const long long c1_ = g.stats ? clock64() : 0;
      const int64_t nk = nd.n, Sk = nd.S;
      const float nkf = __ll2float_rn(nk), Skf = __ll2float_rn(Sk);
      uint32_t* stg = temp;  // the medium levels' partition buffer (>= TGRP * TINY entries)
      const unsigned lt = (1u << lane) - 1u;
      // lane-local best over all (feature, boundary) items: key g, tie = (feature << 16 | rank)
      double lg = -1.0;
      uint32_t ltie = 0xffffffffu, lra = 0, lrb = 0;
      int32_t lnl = 0;
      int64_t lSl = 0;
      if constexpr (LPF) {
        // Lane s scans drawn feature feats[s] (s = lane, lane + 32, ...) serially over the node's own rows: the
        // node's rows in that feature's value order are the set bits of Mf (positions in the tiny root's
        // segment), so the loop runs an times with no staging, no segmented warp scan and no idle positions.
        // Per boundary the fp32 bounds tL <= t <= tU (key_bounds_t); M = warp max of the lower bounds; a lane
        // whose second-largest upper bound is below M evaluates its one candidate directly, any other lane with
        // an upper bound >= M re-walks its features taking the exact S4.3 key where tU >= M.
        // TV 2: every drawn feature's member mask by ballots over the root's segment (lane k tests the row at
        // position k), kept in the warp's scratch (no position table)
        uint64_t* mkw = reinterpret_cast<uint64_t*>(temp + (((uintptr_t)temp >> 2) & 1));  // 8-byte aligned
        if constexpr (TV == 2) {
          static_assert(NWD == 1, "ballot masks cover tiny roots of <= 64 rows");
          for (int u0 = 0; u0 < g.mtry; u0 += 7) {
            uint32_t ev[14];
#pragma unroll
            for (int u = 0; u < 7; ++u) {
              const uint32_t* sg = list + (size_t)feats[min(u0 + u, g.mtry - 1)] * a0 + rlo;
              ev[2 * u] = lane < ra ? sg[lane] : 0u;
              ev[2 * u + 1] = lane + 32 < ra ? sg[lane + 32] : 0u;
            }
#pragma unroll
            for (int u = 0; u < 7; ++u) {
              const int ri0 = rmap[ev[2 * u] & 0xffffu], ri1 = rmap[ev[2 * u + 1] & 0xffffu];
              const uint32_t b0 = __ballot_sync(0xffffffffu, lane < ra && ((nd.mask[0] >> ri0) & 1ull));
              const uint32_t b1 = __ballot_sync(0xffffffffu, lane + 32 < ra && ((nd.mask[0] >> ri1) & 1ull));
              if (lane == 0 && u0 + u < g.mtry) mkw[u0 + u] = ((uint64_t)b1 << 32) | b0;
            }
          }
          __syncwarp();
        }
        auto feat_mask_s = [&](int s, uint64_t (&Mf)[NWD]) {
          if constexpr (TV == 2) {
            Mf[0] = mkw[s];
          } else {
            const uint8_t* pp = ppos + (size_t)feats[s] * a0 + rlo;
            uint64_t m[NWD];
#pragma unroll
            for (int w = 0; w < NWD; ++w) {
              m[w] = nd.mask[w];
              Mf[w] = 0ull;
            }
#pragma unroll 4
            for (int c = 0; c < an; ++c) m_set(Mf, (int)pp[m_pop(m)]);
          }
        };
        float mLt = -1.0f, mU = -1.0f, u2 = -1.0f;
        int bs = -1;
        uint32_t be = 0, ben = 0;
        int32_t bcw = 0;
        int64_t bcs = 0;
        for (int s = lane; s < g.mtry; s += 32) {
          const uint32_t* seg = list + (size_t)feats[s] * a0 + rlo;
          uint64_t Mf[NWD];
          feat_mask_s(s, Mf);
          uint32_t pe = seg[m_pop(Mf)];
          int32_t cw = wl[pe & 0xffffu];
          int64_t cs = wy[pe & 0xffffu];
#pragma unroll 2
          for (int c = 1; c < an; ++c) {
            const uint32_t e = seg[m_pop(Mf)];
            if ((e >> 16) != (pe >> 16)) {
              float tL, tU;
              key_bounds_t(nkf, Skf, nk, cw, cs, tL, tU);
              mLt = fmaxf(mLt, tL);
              if (tU > mU) {
                u2 = mU;
                mU = tU;
                bs = s;
                be = pe;
                ben = e;
                bcw = cw;
                bcs = cs;
              } else {
                u2 = fmaxf(u2, tU);
              }
            }
            cw += wl[e & 0xffffu];
            cs += wy[e & 0xffffu];
            pe = e;
          }
        }
        const float M = warp_max_t(mLt);
        if (mU >= M && mU >= 0.0f && u2 < M) {  // a single candidate on this lane
          lg = split_key(nk, Sk, bcw, bcs);
          ltie = ((uint32_t)feats[bs] << 16) | (be >> 16);
          lnl = bcw;
          lSl = bcs;
          lra = be & 0xffffu;
          lrb = ben & 0xffffu;
        } else if (mU >= M && mU >= 0.0f) {
          for (int s = lane; s < g.mtry; s += 32) {
            const uint32_t* seg = list + (size_t)feats[s] * a0 + rlo;
            uint64_t Mf[NWD];
            feat_mask_s(s, Mf);
            uint32_t pe = seg[m_pop(Mf)];
            int32_t cw = wl[pe & 0xffffu];
            int64_t cs = wy[pe & 0xffffu];
            for (int c = 1; c < an; ++c) {
              const uint32_t e = seg[m_pop(Mf)];
              if ((e >> 16) != (pe >> 16)) {
                float tL, tU;
                key_bounds_t(nkf, Skf, nk, cw, cs, tL, tU);
                if (tU >= M) {
                  const double gk = split_key(nk, Sk, cw, cs);
                  const uint32_t tie = ((uint32_t)feats[s] << 16) | (pe >> 16);
                  if (gk > lg || (gk == lg && tie < ltie)) {
                    lg = gk;
                    ltie = tie;
                    lnl = cw;
                    lSl = cs;
                    lra = pe & 0xffffu;
                    lrb = e & 0xffffu;
                  }
                }
              }
              cw += wl[e & 0xffffu];
              cs += wy[e & 0xffffu];
              pe = e;
            }
          }
        }
        (void)stg;
        (void)lt;
      } else {
      // Features go in groups as large as the staging area holds (ng * an <= sub_temp(A) entries): every drawn
      // feature in ONE group when the node has few distinct rows, so the scan / bound / max passes and their
      // fixed costs run once per node instead of once per TGRP features.
      const int gcap = max(1, sub_temp(g.A) / max(an, 1));
      for (int s0 = 0; s0 < g.mtry;) {
        const long long gqs = g.stats ? clock64() : 0;
        const int ng = min(gcap, g.mtry - s0);
        // stage: the node's entries of each drawn feature, in value order, packed [slot][0..an), TGRP features
        // at a time with all their loads issued before any store (ILP across features); the second half-warp row
        // only when the tiny root has more than 32 rows (warp-uniform).
        for (int u0 = 0; u0 < ng; u0 += TGRP) {
          const int nu = min(TGRP, ng - u0);
          uint32_t ev[2 * TGRP];
          uint8_t ri[2 * TGRP];
          if (ra > 32) {
#pragma unroll
            for (int u = 0; u < TGRP; ++u) {
              const uint32_t* seg = list + (size_t)feats[s0 + u0 + (u < nu ? u : 0)] * a0 + rlo;
              ev[2 * u] = (u < nu) ? seg[lane] : 0u;
              ev[2 * u + 1] = (u < nu && lane + 32 < ra) ? seg[lane + 32] : 0u;
            }
#pragma unroll
            for (int k = 0; k < 2 * TGRP; ++k) ri[k] = rmap[ev[k] & 0xffffu];
#pragma unroll
            for (int u = 0; u < TGRP; ++u) {
              const bool v0 = u < nu && ((nd.mask[0] >> ri[2 * u]) & 1ull);
              const bool v1 = u < nu && lane + 32 < ra && ((nd.mask[0] >> ri[2 * u + 1]) & 1ull);
              const unsigned m0 = __ballot_sync(0xffffffffu, v0), m1 = __ballot_sync(0xffffffffu, v1);
              if (v0) stg[(u0 + u) * an + __popc(m0 & lt)] = ev[2 * u];
              if (v1) stg[(u0 + u) * an + __popc(m0) + __popc(m1 & lt)] = ev[2 * u + 1];
            }
          } else {
#pragma unroll
            for (int u = 0; u < TGRP; ++u) {
              const uint32_t* seg = list + (size_t)feats[s0 + u0 + (u < nu ? u : 0)] * a0 + rlo;
              ev[u] = (u < nu && lane < ra) ? seg[lane] : 0u;
            }
#pragma unroll
            for (int k = 0; k < TGRP; ++k) ri[k] = rmap[ev[k] & 0xffffu];
#pragma unroll
            for (int u = 0; u < TGRP; ++u) {
              const bool v0 = u < nu && lane < ra && ((nd.mask[0] >> ri[u]) & 1ull);
              const unsigned m0 = __ballot_sync(0xffffffffu, v0);
              if (v0) stg[(u0 + u) * an + __popc(m0 & lt)] = ev[u];
            }
          }
        }
        __syncwarp();
        const long long gq0 = g.stats ? clock64() : 0;
        // the ng*an (slot, position) items, K consecutive ones per lane: (A) lane-serial sums of the lane's
        // trailing slot run; one segmented warp scan of those runs; (B) lane-serial prefixes and cheap rigorous
        // bounds gL <= g <= gU at every boundary; M = warp max of the lower bounds (and of the best exact key
        // so far); (C) only lanes holding an item with gU >= M redo their items and take the exact S4.3 key.
        const int total = ng * an;
        const int K = (total + 31) >> 5;
        const int i0 = min(lane * K, total), i1 = min(i0 + K, total);
        const int slot0 = i0 / an, jj0 = i0 - slot0 * an;
        int32_t rw = 0;
        int64_t rsum = 0;
        bool hs = false;
        {
          int jj = jj0;
#pragma unroll 4
          for (int i = i0; i < i1; ++i) {
            if (jj == 0) {
              rw = 0;
              rsum = 0;
              hs = true;
            }
            const uint32_t lr = stg[i] & 0xffffu;
            rw += wl[lr];
            rsum += wy[lr];
            if (++jj == an) jj = 0;
          }
        }
        const long long gq1 = g.stats ? clock64() : 0;
        // segmented inclusive scan over lanes: (v, f) (+) (v', f') = (f' ? v' : v + v', f | f')
        {
          bool f = hs;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const int32_t uw = __shfl_up_sync(0xffffffffu, rw, o);
            const int64_t us = __shfl_up_sync(0xffffffffu, rsum, o);
            const bool uf = __shfl_up_sync(0xffffffffu, f, o);
            if (lane >= o) {
              if (!f) {
                rw += uw;
                rsum += us;
              }
              f = f || uf;
            }
          }
        }
        int32_t cw0 = __shfl_up_sync(0xffffffffu, rw, 1);
        int64_t cs0 = __shfl_up_sync(0xffffffffu, rsum, 1);
        if (lane == 0 || jj0 == 0) {
          cw0 = 0;
          cs0 = 0;
        }
        const long long gq2 = g.stats ? clock64() : 0;
        // the lane's largest upper bound mU with its item (bi, prefix bcw / bcs) and the second largest u2: when
        // u2 < M only item bi can reach the exact-key pass, which then evaluates it directly
        float mL = key_t_lower(lg), mU = -1.0f, u2 = -1.0f;  // fp32 t-space screen
        int bi = -1;
        int32_t bcw = 0;
        int64_t bcs = 0;
        {
          int jj = jj0;
          int32_t cw = cw0;
          int64_t cs = cs0;
#pragma unroll 1
          for (int i = i0; i < i1; ++i) {
            if (jj == 0) {
              cw = 0;
              cs = 0;
            }
            const uint32_t e = stg[i], lr = e & 0xffffu;
            cw += wl[lr];
            cs += wy[lr];
            if (jj + 1 < an && (stg[i + 1] >> 16) != (e >> 16)) {
              float gL, gU;
              key_bounds_t(nkf, Skf, nk, cw, cs, gL, gU);
              mL = fmaxf(mL, gL);
              if (gU > mU) {
                u2 = mU;
                mU = gU;
                bi = i;
                bcw = cw;
                bcs = cs;
              } else {
                u2 = fmaxf(u2, gU);
              }
            }
            if (++jj == an) jj = 0;
          }
        }
        const long long gq3 = g.stats ? clock64() : 0;
        const float M = warp_max_t(mL);
        const long long gq4 = g.stats ? clock64() : 0;
        if (mU >= M && mU >= 0.0f && u2 < M) {  // a single candidate item on this lane
          const uint32_t e = stg[bi], en = stg[bi + 1];
          const double gk = split_key(nk, Sk, bcw, bcs);
          const uint32_t tie = ((uint32_t)feats[s0 + bi / an] << 16) | (e >> 16);
          if (gk > lg || (gk == lg && tie < ltie)) {
            lg = gk;
            ltie = tie;
            lnl = bcw;
            lSl = bcs;
            lra = e & 0xffffu;
            lrb = en & 0xffffu;
          }
        } else if (mU >= M && mU >= 0.0f) {
          int jj = jj0, sl = slot0;
          int32_t cw = cw0;
          int64_t cs = cs0;
          for (int i = i0; i < i1; ++i) {
            if (jj == 0) {
              cw = 0;
              cs = 0;
            }
            const uint32_t e = stg[i], lr = e & 0xffffu;
            cw += wl[lr];
            cs += wy[lr];
            if (jj + 1 < an) {
              const uint32_t en = stg[i + 1];
              if ((en >> 16) != (e >> 16)) {
                float gL, gU;
                key_bounds_t(nkf, Skf, nk, cw, cs, gL, gU);
                if (gU >= M) {
                  const double gk = split_key(nk, Sk, cw, cs);
                  const uint32_t tie = ((uint32_t)feats[s0 + sl] << 16) | (e >> 16);
                  if (gk > lg || (gk == lg && tie < ltie)) {
                    lg = gk;
                    ltie = tie;
                    lnl = cw;
                    lSl = cs;
                    lra = lr;
                    lrb = en & 0xffffu;
                  }
                }
              }
            }
            if (++jj == an) {
              jj = 0;
              ++sl;
            }
          }
        }
        if (g.stats && lane == 0) {
          const long long gq5 = clock64();
          atomicAdd(&g.stats[21], (unsigned long long)(gq0 - gqs));
          atomicAdd(&g.stats[16], (unsigned long long)(gq1 - gq0));
          atomicAdd(&g.stats[17], (unsigned long long)(gq2 - gq1));
          atomicAdd(&g.stats[18], (unsigned long long)(gq3 - gq2));
          atomicAdd(&g.stats[19], (unsigned long long)(gq4 - gq3));
          atomicAdd(&g.stats[20], (unsigned long long)(gq5 - gq4));
        }
        __syncwarp();
        s0 += ng;
      }
      }  // TV == 0
      const long long c2_ = g.stats ? clock64() : 0;
      if (g.stats && lane == 0) { atomicAdd(&g.stats[11], (unsigned long long)(c1_ - c0_)); atomicAdd(&g.stats[12], (unsigned long long)(c2_ - c1_)); }
      const int wlane = warp_argmax_key(gkey(lg), ltie);
      const double bgs = __shfl_sync(0xffffffffu, lg, wlane >= 0 ? wlane : 0);
      const double bg = wlane >= 0 ? bgs : -1.0;
      if (bg > 0.0) {
        const uint32_t tie = __shfl_sync(0xffffffffu, ltie, wlane);
        const int bf = (int)(tie >> 16);
        const uint32_t brk = tie & 0xffffu;
        const int32_t bnl = __shfl_sync(0xffffffffu, lnl, wlane);
        const int64_t bSl = __shfl_sync(0xffffffffu, lSl, wlane);
        const uint32_t bra = __shfl_sync(0xffffffffu, lra, wlane);
        const uint32_t brb = __shfl_sync(0xffffffffu, lrb, wlane);
        // child masks from the winning feature's order: left = rank <= brk
        const uint32_t* seg = list + (size_t)bf * a0 + rlo;
        uint32_t lw[2 * NWD];  // this lane's left rows, by 32-bit word of the mask
#pragma unroll
        for (int w = 0; w < 2 * NWD; ++w) lw[w] = 0u;
        double vl = 0.0, vr = 0.0;
  #pragma unroll
        for (int hh = 0; hh < TT / 32; ++hh) {
          const int k = lane + 32 * hh;
          if (TT > 64 && 32 * hh >= ra) break;  // warp-uniform
          const uint32_t e = k < ra ? seg[k] : 0u;
          const uint32_t lrow = e & 0xffffu;
          const int ri = k < ra ? rmap[lrow] : 0;
          const bool valid = k < ra && m_test(nd.mask, ri);
          const bool left = valid && (e >> 16) <= brk;
#pragma unroll
          for (int w = 0; w < 2 * NWD; ++w) lw[w] |= (left && (ri >> 5) == w) ? 1u << (ri & 31) : 0u;
          if (!DEFER) {
            if (left) vl += wyd[lrow];
            else if (valid) vr += wyd[lrow];
          }
        }
        uint64_t mL[NWD], mR[NWD];
#pragma unroll
        for (int w = 0; w < NWD; ++w) {
          mL[w] = ((uint64_t)__reduce_or_sync(0xffffffffu, lw[2 * w + 1]) << 32) | __reduce_or_sync(0xffffffffu, lw[2 * w]);
          mR[w] = nd.mask[w] & ~mL[w];
        }
        if (!DEFER) {
  #pragma unroll
          for (int o = 16; o > 0; o >>= 1) {
            vl += __shfl_down_sync(0xffffffffu, vl, o);
            vr += __shfl_down_sync(0xffffffffu, vr, o);
          }
        }
        const int nr = nd.n - bnl;
        const bool gl = bnl > g.nodesize && m_popc(mL) >= 2;
        const bool gr = nr > g.nodesize && m_popc(mR) >= 2;
        const double val_l = DEFER ? __longlong_as_double((long long)mL[0]) : __ddiv_rn(vl, (double)bnl);
        const double val_r = DEFER ? __longlong_as_double((long long)mR[0]) : __ddiv_rn(vr, (double)nr);
        // Records: a node's whole record is written by the warp that grows it (this one for nd); a child that
        // stays a leaf gets its record here, a child that is grown further (here or by the warp that takes it
        // from the queue) writes its own -- so no record is written by two warps without a barrier between.
        int lid = 0;
        if (lane == 0) {
          lid = atomicAdd(&s_nloc[nd.id >> 16], 2);
          SRec r;
          r.feature = bf;
          r.left = lid;
          r.count = nd.n;
          r.ra = (uint16_t)bra;
          r.rb = (uint16_t)brb;
          r.value = DEFER ? __longlong_as_double((long long)nd.mask[0]) : nd.value;
          r.drss = ldexp(__ddiv_rn(bg, (double)nd.n), -2 * g.q);
          recs[nd.id & 0xffff] = r;
          if (DEFER) rdef[nd.id & 0xffff] = (uint16_t)rlo;
          SRec c;
          c.feature = -1;
          c.left = -1;
          c.ra = c.rb = 0;
          c.drss = 0.0;
          if (!gl) {
            c.count = bnl;
            c.value = val_l;
            recs[lid] = c;
            if (DEFER) rdef[lid] = (uint16_t)rlo;
          }
          if (!gr) {
            c.count = nr;
            c.value = val_r;
            recs[lid + 1] = c;
            if (DEFER) rdef[lid + 1] = (uint16_t)rlo;
          }
        }
        lid = __shfl_sync(0xffffffffu, lid, 0);
        // child keys on lanes 0 and 1 (computed before the search)
        const uint64_t kl = __shfl_sync(0xffffffffu, ck, 0), kr = __shfl_sync(0xffffffffu, ck, 1);
        TN cl, cr;
        cl.value = val_l;
        cr.value = val_r;
        cl.rlo = cr.rlo = nd.rlo;
        cl.ra = cr.ra = nd.ra;
#pragma unroll
        for (int w = 0; w < NWD; ++w) {
          cl.mask[w] = mL[w];
          cr.mask[w] = mR[w];
        }
        cl.id = (nd.id & ~0xffff) | lid;
        cl.n = bnl;
        cl.S = bSl;
        cl.key = kl;
        cr.id = (nd.id & ~0xffff) | (lid + 1);
        cr.n = nr;
        cr.S = nd.S - bSl;
        cr.key = kr;
        // continue with one child in this warp, hand the sibling to the queue
        if (gl && gr) {
          // the larger child keeps the warp (the longer remaining chain stays off the queue's hand-off latency)
          const bool keep_r = g.tq_bigger_first && m_popc(mR) > m_popc(mL);
          if (lane == 0) tq_push(tq, tq_ready, &s_alloc, &s_pending, keep_r ? cl : cr);
          nd = keep_r ? cr : cl;
          have = true;
        } else if (gl) {
          nd = cl;
          have = true;
        } else if (gr) {
          nd = cr;
          have = true;
        }
      } else if (lane == 0) {  // no positive-gain split (S4.5): the node is a leaf; its record is written here
        SRec r;
        r.feature = -1;
        r.left = -1;
        r.count = nd.n;
        r.ra = r.rb = 0;
        r.value = DEFER ? __longlong_as_double((long long)nd.mask[0]) : nd.value;
        r.drss = 0.0;
        recs[nd.id & 0xffff] = r;
        if (DEFER) rdef[nd.id & 0xffff] = (uint16_t)rlo;
      }

    }
    busy += clock64() - tb0;
    if (lane == 0) atomicSub(&s_pending, 1);
    __syncwarp();
  }
  __syncthreads();
  const long long t_tiny_end = clock64();
  __syncthreads();
  tclk[3] = clock64();
  // ---- flush every packed subtree into its tree's raw pool (sibling pairs stay adjacent)
  if (tid < nr) {
    const int nloc = s_nloc[tid] - 2 * s_off[tid];
    s_gbase[tid] = nloc > 1 ? atomicAdd(&g.pool.nn[s_b[tid]], nloc - 1) : 0;
  }
  __syncthreads();
  for (int l = tid; l < 2 * a0; l += SUB_NT) {
    int r = 0;
    while (r + 1 < nr && 2 * s_off[r + 1] <= l) ++r;
    const int rec0 = 2 * s_off[r];
    if (l >= s_nloc[r]) continue;  // unused record slot of root r
    const int k = l - rec0, gbase = s_gbase[r];
    const SRec rc = recs[l];
    const int64_t gid = (int64_t)s_b[r] * g.pool.cap + (k == 0 ? s_root[r].raw : gbase + k - 1);
    g.pool.feature[gid] = rc.feature;
    g.pool.left[gid] = rc.left >= 0 ? gbase + (rc.left - rec0) - 1 : -1;
    double thr = 0.0;
    if (rc.feature >= 0)
      thr = split_threshold(canon(g.X[(int64_t)rc.feature * g.ldx + grow[rc.ra]]),
                            canon(g.X[(int64_t)rc.feature * g.ldx + grow[rc.rb]]));
    g.pool.thr[gid] = thr;
    g.pool.drss[gid] = rc.drss;
    if (k > 0) {
      g.pool.count[gid] = rc.count;
      double v = rc.value;
      if (DEFER && rdef[l] != 0xffffu) {  // S4.7 node value from the record's row mask over its tiny root
        const int rl = rdef[l];
        uint64_t mk = (uint64_t)__double_as_longlong(rc.value);
        const int nb = __popcll(mk);
        double sw = 0.0;
#pragma unroll 4
        for (int c = 0; c < nb; ++c) {  // countable: the row loads of several members are in flight together
          sw += wyd[list[rl + __ffsll((long long)mk) - 1] & 0xffffu];
          mk &= mk - 1;
        }
        v = __ddiv_rn(sw, (double)rc.count);
      }
      g.pool.value[gid] = v;
    }
  }
  if (g.visits && lane == 0 && nvis) atomicAdd(g.visits, nvis);
  if (g.stats) {
    tclk[4] = clock64();
    if (tid == 0) {
      atomicAdd(&g.stats[0], (unsigned long long)(tclk[1] - tclk[0]));
      atomicAdd(&g.stats[1], (unsigned long long)(tclk[2] - tclk[1]));
      atomicAdd(&g.stats[2], (unsigned long long)(tclk[3] - tclk[2]));
      atomicAdd(&g.stats[3], (unsigned long long)(tclk[4] - tclk[3]));
      atomicAdd(&g.stats[13], (unsigned long long)mclk[0]);
      atomicAdd(&g.stats[14], (unsigned long long)mclk[1]);
      atomicAdd(&g.stats[15], (unsigned long long)mclk[2]);
      atomicAdd(&g.stats[22], (unsigned long long)n_mlev);
      atomicAdd(&g.stats[23], (unsigned long long)mfin);
      atomicAdd(&g.stats[4], (unsigned long long)n_med);
      atomicAdd(&g.stats[5], 1ull);
      atomicAdd(&g.stats[6], (unsigned long long)a0);
      for (int r = 0; r < nr; ++r) atomicAdd(&g.stats[9], (unsigned long long)(s_nloc[r] - 2 * s_off[r]));
    }
    if (lane == 0) {
      atomicAdd(&g.stats[7], (unsigned long long)n_tiny);
      atomicAdd(&g.stats[8], (unsigned long long)(t_tiny_end - tclk[2]));  // busy+idle per warp in tiny phase
      atomicAdd(&g.stats[10], (unsigned long long)busy);
    }
  }
}

__global__ void k_small_a(const LNode* sq, int N, int32_t* a) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < N) a[i] = sq[i].a;
}

// ------------------------------------------------------------------ a11 emit
__global__ void k_emit(Pool pool, const int64_t* out_off, Node16* nodes, int32_t* count, double* value,
                       double* drss) {
  const int b = blockIdx.y;
  const int64_t k = blockIdx.x * (int64_t)NT + threadIdx.x;
  const int32_t nn = pool.nn[b];
  if (k >= nn) return;
  const int64_t r = (int64_t)b * pool.cap + k;
  const int64_t o = out_off[b] + k;
  Node16 nd;
  nd.feature = pool.feature[r];
  nd.left = pool.left[r];
  nd.v = nd.feature >= 0 ? pool.thr[r] : pool.value[r];
  nodes[o] = nd;
  count[o] = pool.count[r];
  value[o] = pool.value[r];
  drss[o] = pool.drss[r];
}

int max_optin_smem() {
  int dev = 0, v = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  return v;
}

template <class T>
void h2d(T* d, const T* h, size_t cnt, cudaStream_t s) {
  BF_CUDA_CHECK(cudaMemcpyAsync(d, h, cnt * sizeof(T), cudaMemcpyHostToDevice, s));
}
template <class T>
void d2h(T* h, const T* d, size_t cnt, cudaStream_t s) {
  BF_CUDA_CHECK(cudaMemcpyAsync(h, d, cnt * sizeof(T), cudaMemcpyDeviceToHost, s));
}

// The node-list work space (E0, E1, Es: the three largest buffers of a fit, GBs each) is kept across bf_fit calls
// and reused when large enough, so consecutive fits of one shape make no allocator calls for it (with torch's
// caching allocator a fragmented cache otherwise sometimes releases and re-allocates them: +0.6 s on a C4 step).
// One fit at a time owns it (a concurrent fit on another thread allocates its own); it is never freed at exit.
// BF_LIST_WORKSPACE=0 allocates per fit.
struct ListWorkspace {
  std::mutex mu;
  uint64_t* buf[3] = {nullptr, nullptr, nullptr};
  size_t cap = 0;  // entries per buffer
  int device = -1;
};
ListWorkspace& list_ws() {
  static ListWorkspace* w = new ListWorkspace();
  return *w;
}

}  // namespace

bool release_list_workspace() {
  ListWorkspace& w = list_ws();
  std::unique_lock<std::mutex> lk(w.mu, std::try_to_lock);
  if (!lk.owns_lock()) return false;
  if (w.cap) {
    cudaDeviceSynchronize();
    for (auto& b : w.buf) {
      dev_free(b, nullptr);
      b = nullptr;
    }
    w.cap = 0;
    w.device = -1;
  }
  return true;
}

namespace {

struct PinnedSummary {
  LevelSummary* h = nullptr;
  PinnedSummary() { BF_CUDA_CHECK(cudaMallocHost(&h, sizeof(LevelSummary) * 2)); }
  ~PinnedSummary() { if (h) cudaFreeHost(h); }
};

int grid_for(int64_t work) { return (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(work, NT), 148 * 16)); }

}  // namespace

// ================================================================== host entry points
void fixed_point_impl(const double* y, int64_t n, int64_t ns, int64_t* yq, int32_t* q_out, cudaStream_t s) {
  const int grid = grid_for(n);
  DBuf<double> part(2 * (size_t)grid, s);
  {
    KScope ks_("k_minmax", s, 0.0);
    k_minmax<<<grid, NT, 0, s>>>(y, n, part.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  std::vector<double> hp(2 * (size_t)grid);
  d2h(hp.data(), part.p, hp.size(), s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  double mn = INFINITY, mx = -INFINITY;
  for (int i = 0; i < grid; ++i) {
    mn = std::fmin(mn, hp[2 * i]);
    mx = std::fmax(mx, hp[2 * i + 1]);
  }
  BF_REQUIRE(std::isfinite(mn) && std::isfinite(mx), BF_ENONFINITE, "non-finite y");
  volatile double h0 = 0.5 * mn, h1 = 0.5 * mx;  // S2: c = RN(RN(0.5 min) + RN(0.5 max))
  const double c = h0 + h1;
  {
    KScope ks_("k_absdev_max", s, 0.0);
    k_absdev_max<<<grid, NT, 0, s>>>(y, n, c, part.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  d2h(hp.data(), part.p, (size_t)grid, s);
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  double R = 0.0;
  for (int i = 0; i < grid; ++i) R = std::fmax(R, hp[i]);
  BF_REQUIRE(std::isfinite(R), BF_ERANGE, "y range overflows");
  int q = 0, zero = 0;
  if (R == 0.0) {
    zero = 1;
  } else {
    int e = 0;
    std::frexp(R, &e);
    int sbits = 0;
    for (uint64_t v = (uint64_t)ns; v; v >>= 1) ++sbits;
    q = 62 - sbits - e;
  }
  {
    KScope ks_("k_yq", s, 0.0);
    k_yq<<<grid, NT, 0, s>>>(y, n, c, q, zero, yq);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  *q_out = q;
}

void bootstrap_impl(uint64_t seed, int32_t t0, int32_t ntrees, int64_t n, int64_t ns, int32_t replace, int32_t* w,
                    cudaStream_t s) {
  if (ntrees <= 0) return;
  const int64_t tot = n * ntrees;
  if (!replace) {
    {
      KScope ks_("k_fill_i32", s, 0.0);
      k_fill_i32<<<grid_for(tot), NT, 0, s>>>(w, tot, 1);
    }
    BF_CUDA_CHECK(cudaGetLastError());
    return;
  }
  BF_CUDA_CHECK(cudaMemsetAsync(w, 0, sizeof(int32_t) * tot, s));
  dim3 grid((unsigned)ceil_div(ceil_div(ns, 2), NT), (unsigned)ntrees);
  {
    KScope ks_("k_bootstrap", s, 0.0);
    k_bootstrap<<<grid, NT, 0, s>>>(seed, t0, n, ns, w);
  }
  BF_CUDA_CHECK(cudaGetLastError());
}

struct PhaseTimer {  // BF_FIT_TIMING=1: host wall time per fit phase (stream-synchronised)
  bool on;
  cudaStream_t s;
  double t0, last;
  std::vector<std::pair<std::string, double>> acc;
  static double now() {
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return ts.tv_sec + ts.tv_nsec * 1e-9;
  }
  explicit PhaseTimer(cudaStream_t st) : on(getenv("BF_FIT_TIMING") != nullptr), s(st) { t0 = last = now(); }
  void mark(const char* name) {
    if (!on) return;
    cudaStreamSynchronize(s);
    const double t = now();
    for (auto& kv : acc)
      if (kv.first == name) {
        kv.second += t - last;
        last = t;
        return;
      }
    acc.emplace_back(name, t - last);
    last = t;
  }
  ~PhaseTimer() {
    if (!on) return;
    fprintf(stderr, "[fit timing] total %.1f ms:", (now() - t0) * 1e3);
    for (auto& kv : acc) fprintf(stderr, " %s=%.1f", kv.first.c_str(), kv.second * 1e3);
    fprintf(stderr, "\n");
  }
};

void fit_impl(const double* X_in, int64_t ldx, const double* y_in, int64_t n, int32_t p, const bf_params& prm0,
              cudaStream_t s, bf_forest** out) {
  PhaseTimer ptm(s);
  bf_params prm = prm0;
  BF_REQUIRE(prm.ntree >= 1 && prm.nodesize >= 1, BF_EINVAL, "bf_fit: ntree >= 1 and nodesize >= 1 required");
  if (prm.tree_end < 0) prm.tree_end = prm.ntree;  // whole forest; (b, b) is an honoured empty range
  BF_REQUIRE(prm.tree_begin >= 0 && prm.tree_end <= prm.ntree && prm.tree_begin <= prm.tree_end, BF_EINVAL,
             "bf_fit: bad tree range");
  const int mtry = prm.mtry ? prm.mtry : std::max(p / 3, 1);
  BF_REQUIRE(mtry >= 1 && mtry <= p, BF_EINVAL, "bf_fit: mtry not in [1, p]");
  BF_REQUIRE(p <= 32767, BF_ENOTIMPL, "bf_fit: p > 32767");
  BF_REQUIRE(n < MAX_ROWS, BF_ENOTIMPL, "bf_fit: n >= 2^24 rows (24-bit row/rank fields of the list entries)");
  const int64_t ns = prm.sampsize ? prm.sampsize : n;
  BF_REQUIRE(ns >= 1 && ns < (int64_t(1) << 31), BF_ERANGE, "bf_fit: sampsize out of range");
  BF_REQUIRE(prm.replace || ns == n, BF_ENOTIMPL, "bf_fit: replace = 0 needs sampsize == n (reading R20)");

  InStage Xs(X_in, sizeof(double) * (size_t)(ldx * (p - 1) + n), s);
  InStage ys(y_in, sizeof(double) * (size_t)n, s);
  const double* X = (const double*)Xs.dptr;
  const double* y = (const double*)ys.dptr;

  // ---- a1 validate
  {
    DBuf<int> bad(1, s);
    BF_CUDA_CHECK(cudaMemsetAsync(bad.p, 0, sizeof(int), s));
    {
      KScope ks_("k_validate", s, 0.0);
      k_validate<<<grid_for(n * p + n), NT, 0, s>>>(X, ldx, n, p, y, bad.p);
    }
    BF_CUDA_CHECK(cudaGetLastError());
    int hb = 0;
    d2h(&hb, bad.p, 1, s);
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
    BF_REQUIRE(hb == 0, BF_ENONFINITE, "bf_fit: NaN/Inf in X or y");
  }
  ptm.mark("validate");
  // ---- a2 fixed point
  DBuf<int64_t> yq(n, s);
  int32_t q = 0;
  fixed_point_impl(y, n, ns, yq.p, &q, s);

  // ---- a3 presort (hand-written segmented radix sort of all p features, prims.cu)
  DBuf<uint64_t> srt((size_t)p * n, s);
  DBuf<double> uniq((size_t)p * n, s);
  {
    const int64_t tot = (int64_t)p * n;
    DBuf<uint64_t> k0(tot, s), k1(tot, s);
    DBuf<uint32_t> v0(tot, s), v1(tot, s);
    {
      KScope ks_("k_sort_keys", s, (double)tot * 20.0);
      k_sort_keys<<<grid_for(tot), NT, 0, s>>>(X, ldx, n, p, k0.p, v0.p);
    }
    BF_CUDA_CHECK(cudaGetLastError());
    uint32_t* rows = nullptr;
    const uint64_t* ks = radix_sort_u64(k0.p, k1.p, v0.p, v1.p, n, p, s, &rows);
    uint32_t* fl = rows == v0.p ? v1.p : v0.p;  // the value buffer not holding the sorted rows
    uint64_t* rk64 = const_cast<uint64_t*>(ks == k0.p ? k1.p : k0.p);
    uint32_t* rk = reinterpret_cast<uint32_t*>(rk64);  // scratch: the key buffer not holding the sorted keys
    {
      KScope ks_("k_rank_flags", s, 0.0);
      k_rank_flags<<<grid_for(tot), NT, 0, s>>>(ks, n, p, fl);
    }
    scan_inclusive(fl, rk, tot, s);
    {
      KScope ks_("k_fill_sorted", s, 0.0);
      k_fill_sorted<<<grid_for(tot), NT, 0, s>>>(X, ldx, rows, rk, n, p, srt.p, uniq.p);
    }
    BF_CUDA_CHECK(cudaGetLastError());
  }

  ptm.mark("presort");
  // ---- sizing: subtree capacity A and trees in flight B
  const int smax = std::min(std::min(std::min(dyn_smem_limit(k_subtree<0, 64, 0>), dyn_smem_limit(k_subtree<1, 64, 0>)),
                                     std::min(std::min(dyn_smem_limit(k_subtree<1, 128, 0>), dyn_smem_limit(k_subtree<3, 64, 0>)),
                                              dyn_smem_limit(k_subtree<3, 128, 0>))),
                            std::min(std::min(dyn_smem_limit(k_subtree<2, 64, 0>), dyn_smem_limit(k_subtree<2, 64, 4>)),
                                     dyn_smem_limit(k_subtree<2, 64, 2>)));
  int A = 2;
  // tiny-node search (BF_TINY_V): 3 = lane per drawn feature, member masks from a position table built per tiny
  // root by the warp that takes the root (default); 2 = masks by ballots; 1 = position table built for all tiny
  // roots at the phase start; 0 = staged (slot, position) items scanned by the whole warp.  Measured per 200 C4
  // trees: 452 / 484 / 526 / 600 ms.  Largest tiny root 64 rows (default) or 128 (BF_TINY_MAX=128 with TV 1;
  // slower: the longer tiny chains outweigh the shorter medium phase)
  static const int tiny_v = getenv("BF_TINY_V") ? atoi(getenv("BF_TINY_V")) : 3;
  static const int tiny_max =
      ((tiny_v == 1 || tiny_v == 3) && getenv("BF_TINY_MAX") && atoi(getenv("BF_TINY_MAX")) == 128) ? 128 : 64;
  while (A < 1024 && subtree_smem(A + 1, p, tiny_max) <= (size_t)smax) ++A;  // load 2 holds <= 32 chunks of 32
  BF_REQUIRE(subtree_smem(2, p, tiny_max) <= (size_t)smax, BF_ENOTIMPL,
             "bf_fit: p too large for the shared-memory subtree kernel");
  if (prm.small_node_max > 0) A = std::max(2, std::min(A, prm.small_node_max));

  const int32_t T_loc = prm.tree_end - prm.tree_begin;
  const int64_t cap_nodes = 2 * n + 1;
  const size_t per_tree = (size_t)3 * p * n * 8 + (size_t)n * (4 + 16 + 1 + 2) +
                          (size_t)cap_nodes * (4 + 4 + 4 + 8 + 8 + 8) + (size_t)n * 48 / 2;
  int B = prm.trees_in_flight;
  if (B <= 0) {
    size_t fr = 0, tot = 0;
    BF_CUDA_CHECK(cudaMemGetInfo(&fr, &tot));
    // free memory as the allocator in use sees it: the driver's, or the caller's hint (bf_set_memory_budget:
    // the torch caching allocator's cached-but-unused blocks count as free)
    if (memory_budget() > 0) fr = (size_t)memory_budget();
    {  // a held list work space is this fit's memory too
      int dv_ = 0;
      cudaGetDevice(&dv_);
      if (list_ws().device == dv_) fr += list_ws().cap * 3 * sizeof(uint64_t);
    }
    const size_t budget = fr / 2;
    B = (int)std::max<size_t>(1, std::min<size_t>(budget / std::max<size_t>(per_tree, 1), 256));
    // Large trees: the split-scan and partition CTAs are bound to trees (148 / B CTAs per tree), so a level
    // lasts as long as the tree with the fewest CTAs per unit of work.  Keep that count even: B = SMs / 4
    // (4 partition CTAs per tree) when memory allows, else at most SMs / 7 (ragged 7-8 CTAs per tree).
    if (n >= 65536) {
      int nsm_ = 0, dv_ = 0;
      cudaGetDevice(&dv_);
      cudaDeviceGetAttribute(&nsm_, cudaDevAttrMultiProcessorCount, dv_);
      nsm_ = std::max(nsm_, 8);
      B = B >= nsm_ / 4 ? nsm_ / 4 : std::min(B, nsm_ / 7);
    }
  }
  B = std::max(1, std::min(B, std::max(T_loc, 1)));
  if (ptm.on) fprintf(stderr, "[fit timing] trees in flight B = %d (budget %.1f GB)\n", B, memory_budget() / 1e9);

  bf_forest* F = new bf_forest();
  F->info.n = n;
  F->info.p = p;
  F->info.ntree_total = prm.ntree;
  F->info.tree_begin = prm.tree_begin;
  F->info.tree_end = prm.tree_end;
  F->info.q = q;
  F->info.mtry = mtry;
  F->info.nodesize = prm.nodesize;
  F->info.replace = prm.replace;
  F->info.sampsize = ns;
  F->info.seed = prm.seed;
  cudaGetDevice(&F->device);
  F->tree_off.assign((size_t)T_loc + 1, 0);

  struct Chunk {
    DBuf<Node16> nodes;
    DBuf<int32_t> count;
    DBuf<double> value, drss;
    int64_t total = 0;
  };
  std::vector<Chunk> chunks;

  try {
    ptm.mark("setup");
    // ---- batch buffers
    DBuf<int32_t> w((size_t)B * n, s);
    DBuf<int32_t> wmax(1, s);
    BF_CUDA_CHECK(cudaMemsetAsync(wmax.p, 0, sizeof(int32_t), s));
    DBuf<uint8_t> side((size_t)B * n, s);
    DBuf<int32_t> pf((size_t)B * cap_nodes, s), pl((size_t)B * cap_nodes, s), pc((size_t)B * cap_nodes, s),
        pnn(B, s);
    DBuf<double> pt((size_t)B * cap_nodes, s), pv((size_t)B * cap_nodes, s), pd((size_t)B * cap_nodes, s);
    Pool pool{pf.p, pl.p, pc.p, pt.p, pv.p, pd.p, pnn.p, cap_nodes};
    DBuf<int32_t> a_root(B, s), kind_d(B, s), lidx_d(B, s), sidx_d(B, s);
    DBuf<unsigned long long> S_root(B, s);
    DBuf<double> sy_root(B, s);
    DBuf<int64_t> base_d(B, s), emit_off(B, s);
    const int64_t cap_level = (int64_t)B * n / (A + 1) + B + 1;
    const int64_t cap_small = (int64_t)B * n / 2 + B + 1;
    DBuf<LNode> ncur(cap_level, s), nnext(cap_level, s), sq(cap_small, s);
    DBuf<int32_t> feat(cap_level * mtry, s);
    DBuf<int16_t> fyscr(cap_level * p, s);
    DBuf<Rec> rec(cap_level * mtry, s);
    DBuf<Split> split(cap_level, s);
    DBuf<Child> child(2 * cap_level, s);
    DBuf<uint64_t> packL(2 * cap_level, s), packS(2 * cap_level, s), scanL(2 * cap_level, s), scanS(2 * cap_level, s);
    DBuf<LevelSummary> dsum(1, s);
    PinnedSummary hs;
    // piece decomposition of the winning segments (k_dest_bits), sized for the largest level of a batch
    const int64_t cap_pieces = (int64_t)B * n / PIECE + cap_level + 1;
    DBuf<int32_t> pcnt(cap_level, s), poff(cap_level, s), pmap(cap_pieces, s), ptot(1, s);
    DBuf<double> csum(2 * cap_level, s);
    // partition work items (at most p per node)
    DBuf<int32_t> icnt(cap_level + 1, s), ioff(cap_level + 1, s);
    DBuf<int2> imap(cap_level * p, s);
    auto piece_setup = [&](int mode, int nitems, int div, const LNode* nodes, const Split* sp, const Child* ch,
                           int32_t* cnt, int32_t* off, int32_t* map, int32_t* tot, cudaStream_t st) {
      {
        KScope ks_("k_piece_count", st, 0.0);
        k_piece_count<<<(unsigned)ceil_div(nitems, 256), 256, 0, st>>>(mode, nitems, div, nodes, sp, ch, cnt);
      }
      scan_exclusive(cnt, off, nitems, st);
      {
        KScope ks_("k_piece_map", st, 0.0);
        k_piece_map<<<(unsigned)ceil_div(nitems, 256), 256, 0, st>>>(nitems, cnt, off, map, tot);
      }
    };
    int nsm = 0, dev_id = 0;
    cudaGetDevice(&dev_id);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev_id);
    // tree-affine kernels
    const int64_t nw = (n + 31) / 32;
    DBuf<uint32_t> sideb((size_t)B * nw, s);
    DBuf<int32_t> tlo(B, s), thi(B, s), act(B, s), nact(1, s);
    static const int scan_tsv = getenv("BF_SCAN_TSV") ? atoi(getenv("BF_SCAN_TSV")) : 9;
    auto scan_kern = scan_tsv == 5 ? k_split_scan_tree<5, 6> : scan_tsv == 7 ? k_split_scan_tree<7, 5> : k_split_scan_tree<9, 4>;
    const size_t tscan_smem = sizeof(uint64_t) * 2 * ((size_t)SNT * (scan_tsv == 5 ? 5 : scan_tsv == 7 ? 7 : 9) + 4);
    const size_t tpart_base = sizeof(uint64_t) * (size_t)TPG * (TPNS * (TPUNIT + 2));
    const int smem_optin = dyn_smem_limit(k_partition_tree);
    const bool bm_smem = getenv("BF_PART_L2") == nullptr && tpart_base + (size_t)nw * 4 <= (size_t)smem_optin;
    const size_t tpart_smem = tpart_base + (bm_smem ? (size_t)nw * 4 : 0);
    BF_CUDA_CHECK(cudaFuncSetAttribute(scan_kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tscan_smem));
    int occ_ts = 0, occ_tp = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_ts, scan_kern, SNT, tscan_smem);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_tp, k_partition_tree, TPNT, tpart_smem);
    const unsigned grid_tscan = (unsigned)std::max(1, occ_ts * nsm), grid_tpart = (unsigned)std::max(1, occ_tp * nsm);
    DBuf<uint64_t> E0, E1, Es;  // per-fit list buffers (when the shared work space is not used)
    uint64_t *pE0 = nullptr, *pE1 = nullptr, *pEs = nullptr;
    static const bool ws_on = !(getenv("BF_LIST_WORKSPACE") && getenv("BF_LIST_WORKSPACE")[0] == '0');
    std::unique_lock<std::mutex> wsl(list_ws().mu, std::defer_lock);
    const bool use_ws = ws_on && wsl.try_lock() && (list_ws().device < 0 || list_ws().device == dev_id);
    std::vector<int32_t> h_sa;  // distinct rows of the batch's small roots (subtree packing)
    size_t E_cap = 0;

    ptm.mark("alloc");
    for (int tb = prm.tree_begin; tb < prm.tree_end; tb += B) {
      const int Bc = std::min(B, prm.tree_end - tb);
      // ---- a4 bootstrap + payload + root sums
      bootstrap_impl(prm.seed, tb, Bc, n, ns, prm.replace, w.p, s);
      BF_CUDA_CHECK(cudaMemsetAsync(a_root.p, 0, sizeof(int32_t) * Bc, s));
      BF_CUDA_CHECK(cudaMemsetAsync(S_root.p, 0, sizeof(unsigned long long) * Bc, s));
      BF_CUDA_CHECK(cudaMemsetAsync(sy_root.p, 0, sizeof(double) * Bc, s));
      {
        KScope ks_("k_payload", s, 0.0);
        k_payload<<<dim3((unsigned)ceil_div(n, NT), Bc), NT, 0, s>>>(w.p, yq.p, y, n, wmax.p, a_root.p, S_root.p,
                                                                    sy_root.p);
      }
      BF_CUDA_CHECK(cudaGetLastError());
      std::vector<int32_t> ha(Bc), hk(Bc), hl(Bc), hsx(Bc);
      std::vector<int64_t> hbase(Bc);
      int32_t hwmax = 0;
      d2h(ha.data(), a_root.p, Bc, s);
      d2h(&hwmax, wmax.p, 1, s);
      BF_CUDA_CHECK(cudaStreamSynchronize(s));
      BF_REQUIRE(hwmax <= 0xffff, BF_ERANGE, "bf_fit: a bootstrap multiplicity exceeds 65535");
      int64_t offL = 0, offS = 0;
      int nL = 0, nS = 0;
      for (int b = 0; b < Bc; ++b) {
        hl[b] = hsx[b] = -1;
        hbase[b] = 0;
        if (ns <= prm.nodesize || ha[b] < 2) {
          hk[b] = KIND_LEAF;
        } else if (ha[b] <= A) {
          hk[b] = KIND_SMALL;
          hbase[b] = offS;
          offS += (int64_t)p * ha[b];
          hsx[b] = nS++;
        } else {
          hk[b] = KIND_LARGE;
          hbase[b] = offL;
          offL += (int64_t)p * ha[b];
          hl[b] = nL++;
        }
      }
      // total entries of the batch: every level and the small area fit in sum_b p * a_b
      size_t need = 0;
      for (int b = 0; b < Bc; ++b) need += (size_t)p * ha[b];
      need = std::max<size_t>(need, 1);
      if (need > E_cap) {  // 3% headroom: later batches (sum of in-bag rows varies by ~0.1%) reuse the buffers
        const size_t cap = need + need / 32 + 16;
        if (use_ws) {
          ListWorkspace& w = list_ws();
          if (w.cap < cap) {
            for (auto& b : w.buf) {
              dev_free(b, s);
              b = nullptr;
            }
            w.cap = 0;
            for (auto& b : w.buf) b = (uint64_t*)dev_alloc(cap * sizeof(uint64_t), s);
            w.cap = cap;
            w.device = dev_id;
          }
          pE0 = w.buf[0];
          pE1 = w.buf[1];
          pEs = w.buf[2];
          E_cap = w.cap - 16;
        } else {
          E0.alloc(cap, s);
          E1.alloc(cap, s);
          Es.alloc(cap, s);
          pE0 = E0.p;
          pE1 = E1.p;
          pEs = Es.p;
          E_cap = cap - 16;
        }
      }
      h2d(kind_d.p, hk.data(), Bc, s);
      h2d(lidx_d.p, hl.data(), Bc, s);
      h2d(sidx_d.p, hsx.data(), Bc, s);
      h2d(base_d.p, hbase.data(), Bc, s);
      {
        KScope ks_("k_roots", s, 0.0);
        k_roots<<<(unsigned)ceil_div(Bc, 128), 128, 0, s>>>(Bc, ns, prm.nodesize, a_root.p, S_root.p, sy_root.p,
                                                            kind_d.p, base_d.p, pool, ncur.p, lidx_d.p, sq.p, sidx_d.p);
      }
      BF_CUDA_CHECK(cudaGetLastError());
      // ---- a5 root lists
      {
        const int nchunk = (int)ceil_div(n, LCH);
        DBuf<int32_t> cnt((size_t)Bc * p * nchunk, s);
        const int Bp = (Bc + LTG - 1) / LTG * LTG;
        DBuf<uint16_t> wpk((size_t)n * Bp, s);
        {
          KScope ks_("k_w_pack", s, (double)n * Bc * 4.0 + (double)n * Bp * 2.0);
          k_w_pack<<<(unsigned)ceil_div(n, NT), NT, 0, s>>>(w.p, n, Bc, Bp, wpk.p);
        }
        dim3 grid((unsigned)nchunk, (unsigned)p, (unsigned)(Bp / LTG));
        {
          KScope ks_("k_list_count", s, 0.0);
          k_list_count<<<grid, NT, 0, s>>>(srt.p, n, wpk.p, Bp, kind_d.p, nchunk, Bc, cnt.p);
        }
        {
          KScope ks_("k_list_prefix", s, 0.0);
          k_list_prefix<<<(unsigned)ceil_div((int64_t)Bc * p, 128), 128, 0, s>>>(cnt.p, Bc * p, nchunk);
        }
        {
          KScope ks_("k_list_scatter", s, 0.0);
          k_list_scatter<<<grid, NT, 0, s>>>(srt.p, n, wpk.p, Bp, kind_d.p, base_d.p, a_root.p, nchunk, Bc, cnt.p, pE0,
                                            pEs);
        }
        BF_CUDA_CHECK(cudaGetLastError());
        // presort chunk read once per tree group + one 32 B weight gather per (entry, group) + written entries
        prof_add_bytes("k_list_scatter", (double)(Bp / LTG) * n * p * 40.0 + (double)(offL + offS) * 8.0);
      }
      ptm.mark("boot+lists");
      LevelSummary ls{};
      ls.nnext = nL;
      ls.nsmall = nS;
      ls.small_elems = offS;
      ls.next_elems = offL;
      h2d(dsum.p, &ls, 1, s);
      // ---- global phase
      int N = nL;
      int64_t cur_elems = offL;  // sum of p*a over the level's nodes
      uint64_t* Ec = pE0;
      uint64_t* En = pE1;
      LNode* nc = ncur.p;
      LNode* nx = nnext.p;
      while (N > 0) {
        const int64_t cur_a = cur_elems / p;  // sum of a over the level's nodes
        {
          KScope ks_("k_mtry", s, 0.0);
          k_mtry<<<(unsigned)ceil_div(N, 128), 128, 0, s>>>(nc, N, p, mtry, prm.seed, tb, feat.p, fyscr.p);
        }
        static const bool lvl_timing = getenv("BF_LEVEL_TIMING") != nullptr;
        cudaEvent_t lev[4];
        if (lvl_timing) {
          for (auto& e : lev) cudaEventCreate(&e);
          cudaEventRecord(lev[0], s);
        }
        BF_CUDA_CHECK(cudaMemsetAsync(tlo.p, 0, sizeof(int32_t) * Bc, s));
        BF_CUDA_CHECK(cudaMemsetAsync(thi.p, 0, sizeof(int32_t) * Bc, s));
        {
          KScope ks_("k_tree_ranges", s, 0.0, 2);
          k_tree_ranges<<<(unsigned)ceil_div(N, 256), 256, 0, s>>>(N, nc, tlo.p, thi.p);
          k_active_trees<<<1, 256, 0, s>>>(Bc, tlo.p, thi.p, act.p, nact.p);
        }
        {  // ---- a7 split search: tree-affine CTAs own whole (node, drawn feature) items
          TScanArgs ga{nc, feat.p, mtry, Bc, Ec, yq.p, tlo.p, thi.p, rec.p, act.p, nact.p};
          KScope ks_("k_split_scan_tree", s, 0.0);
          scan_kern<<<grid_tscan, SNT, tscan_smem, s>>>(ga);
        }
        if (lvl_timing) cudaEventRecord(lev[1], s);
        {
          KScope ks_("k_finalize", s, 0.0);
          k_finalize<<<(unsigned)ceil_div(N, 128), 128, 0, s>>>(nc, N, feat.p, rec.p, mtry, uniq.p, n, prm.nodesize, A,
                                                               q, prm.seed, tb, pool, split.p, child.p, packL.p, packS.p, dsum.p);
        }
        BF_CUDA_CHECK(cudaGetLastError());
        const int N2 = 2 * N;
        scan_exclusive(packL.p, scanL.p, N2, s);
        scan_exclusive(packS.p, scanS.p, N2, s);
        {
          KScope ks_("k_child_place", s, 0.0);
          k_child_place<<<(unsigned)ceil_div(N2, 128), 128, 0, s>>>(N2, p, nc, child.p, scanL.p, scanS.p, nx, sq.p,
                                                                    dsum.p);
        }
        // ---- a9/a10 goes-right flags and child values over pieces of the winning segments
        piece_setup(1, N, 1, nc, split.p, child.p, pcnt.p, poff.p, pmap.p, ptot.p, s);
        BF_CUDA_CHECK(cudaMemsetAsync(csum.p, 0, sizeof(double) * 2 * (size_t)N, s));
        // goes-right bitmap cleared per level (n/8 bytes per tree), so only right-going rows need an atomic
        BF_CUDA_CHECK(cudaMemsetAsync(sideb.p, 0, sizeof(uint32_t) * (size_t)Bc * nw, s));
        {
          DestArgs ga{nc, split.p, Ec, y, n, side.p, poff.p, pmap.p, ptot.p, csum.p};
          KScope ks_("k_dest_bits", s, 0.0);
          k_dest_bits<<<(unsigned)(cur_a / PIECE + N + 1), NT, 0, s>>>(ga, sideb.p, nw);
        }
        {
          KScope ks_("k_child_values", s, 0.0);
          k_child_values<<<(unsigned)ceil_div(N, 128), 128, 0, s>>>(N, split.p, csum.p, nc, pool);
        }
        if (lvl_timing) cudaEventRecord(lev[2], s);
        // ---- a9 partition: tree-affine CTAs own whole items; goes-right bitmap in shared memory
        {
          KScope ks_("k_part_items", s, 0.0);
          k_part_items_count<<<(unsigned)ceil_div(N + 1, 256), 256, 0, s>>>(N, p, nc, split.p, child.p, icnt.p);
          scan_exclusive(icnt.p, ioff.p, N + 1, s);
          k_part_items_map<<<(unsigned)ceil_div(N, 256), 256, 0, s>>>(N, p, nc, icnt.p, ioff.p, imap.p);
        }
        {
          TPartArgs ga{nc, split.p, child.p, p, Bc, Ec, sideb.p, nw, bm_smem ? 1 : 0, En, pEs, tlo.p, thi.p, ioff.p, imap.p,
                       act.p, nact.p};
          KScope ks_("k_partition_tree", s, 0.0);
          k_partition_tree<<<grid_tpart, TPNT, tpart_smem, s>>>(ga);
        }
        if (lvl_timing) cudaEventRecord(lev[3], s);
        {
          KScope ks_("k_commit", s, 0.0);
          k_commit<<<1, 1, 0, s>>>(N2, packL.p, scanL.p, packS.p, scanS.p, p, dsum.p, hs.h);
        }
        BF_CUDA_CHECK(cudaGetLastError());
        BF_CUDA_CHECK(cudaStreamSynchronize(s));
        {  // algorithmic bytes
          const double sa = (double)hs.h->split_a;
          prof_add_bytes("k_split_scan_tree", (double)cur_a * mtry * 16.0);
          prof_add_bytes("k_dest_bits", sa * 17.0);
          prof_add_bytes("k_partition_tree", sa * p * 17.0);
        }
        if (lvl_timing) {
          float ms1 = 0, ms2 = 0, ms3 = 0;
          cudaEventElapsedTime(&ms1, lev[0], lev[1]);
          cudaEventElapsedTime(&ms2, lev[1], lev[2]);
          cudaEventElapsedTime(&ms3, lev[2], lev[3]);
          fprintf(stderr, "[level] N=%d entries/feature=%lld split_a=%llu scan=%.3f mid=%.3f part=%.3f ms  scanGB/s=%.0f partGB/s=%.0f\n", N,
                  (long long)cur_a, (unsigned long long)hs.h->split_a, ms1, ms2, ms3,
                  (double)cur_a * mtry * 16.0 / (ms1 * 1e6), (double)hs.h->split_a * p * 17.0 / (ms3 * 1e6));
          for (auto& e : lev) cudaEventDestroy(e);
        }
        cur_elems = hs.h->next_elems;
        N = hs.h->nnext;
        std::swap(Ec, En);
        std::swap(nc, nx);
      }
      ptm.mark("global_levels");
      // ---- subtree phase
      {
        d2h(&ls, dsum.p, 1, s);
        BF_CUDA_CHECK(cudaStreamSynchronize(s));
        if (ls.nsmall > 0) {
          prof_add_bytes("k_subtree", (double)ls.small_elems * 8.0 + (double)ls.small_elems / p * 26.0);
          // Pack small roots into CTAs (distinct rows adding up to <= A, at most MAXR per CTA): the largest
          // remaining root first, topped up with the smallest ones, so every CTA has several independent subtrees
          // whose tiny-node tails overlap (BF_SUBTREE_PACK=0: one root per CTA).
          static const bool pack = !(getenv("BF_SUBTREE_PACK") && getenv("BF_SUBTREE_PACK")[0] == '0');
          const int nsm_roots = ls.nsmall;
          if ((int)h_sa.size() < nsm_roots) h_sa.resize(nsm_roots);
          DBuf<int32_t> d_sa(nsm_roots, s), d_perm(nsm_roots, s), d_gst(nsm_roots + 1, s);
          {
            KScope ks_("k_small_a", s, 0.0);
            k_small_a<<<(unsigned)ceil_div(nsm_roots, 256), 256, 0, s>>>(sq.p, nsm_roots, d_sa.p);
          }
          d2h(h_sa.data(), d_sa.p, nsm_roots, s);
          BF_CUDA_CHECK(cudaStreamSynchronize(s));
          std::vector<int32_t> perm(nsm_roots), gst;
          for (int i = 0; i < nsm_roots; ++i) perm[i] = i;
          if (pack) {
            // descending by distinct rows, ties by index: a counting sort over a in [0, A] (O(roots + A) on
            // the host; a comparison sort of ~80K roots per batch cost ~7 ms)
            {
              std::vector<int32_t> cnt_a((size_t)A + 2, 0);
              for (int i = 0; i < nsm_roots; ++i) ++cnt_a[(size_t)(A - std::min(h_sa[i], A))];
              int run = 0;
              for (size_t v = 0; v < cnt_a.size(); ++v) {
                const int c = cnt_a[v];
                cnt_a[v] = run;
                run += c;
              }
              for (int i = 0; i < nsm_roots; ++i) perm[cnt_a[(size_t)(A - std::min(h_sa[i], A))]++] = i;
            }
            std::vector<int32_t> order;
            order.reserve(nsm_roots);
            int lo_i = 0, hi_i = nsm_roots - 1;
            while (lo_i <= hi_i) {
              gst.push_back((int32_t)order.size());
              int sum = h_sa[perm[lo_i]], cnt = 1;
              order.push_back(perm[lo_i++]);
              while (lo_i <= hi_i && cnt < MAXR && sum + h_sa[perm[hi_i]] <= A) {
                sum += h_sa[perm[hi_i]];
                ++cnt;
                order.push_back(perm[hi_i--]);
              }
            }
            perm.swap(order);
          } else {
            for (int i = 0; i < nsm_roots; ++i) gst.push_back(i);
          }
          const int ngroups = (int)gst.size();
          gst.push_back(nsm_roots);
          h2d(d_perm.p, perm.data(), nsm_roots, s);
          h2d(d_gst.p, gst.data(), ngroups + 1, s);
          SubArgs ga;
          ga.sq = sq.p;
          ga.gperm = d_perm.p;
          ga.gstart = d_gst.p;
          ga.Es = pEs;
          ga.yq = yq.p;
          ga.y = y;
          ga.X = X;
          ga.ldx = ldx;
          ga.n = n;
          ga.p = p;
          ga.mtry = mtry;
          ga.nodesize = prm.nodesize;
          ga.q = q;
          ga.A = A;
          ga.seed = prm.seed;
          ga.t0 = tb;
          ga.pool = pool;
          ga.stats = nullptr;
          ga.visits = nullptr;
          DBuf<unsigned long long> vis;
          if (prof_enabled()) {
            vis.alloc(1, s);
            BF_CUDA_CHECK(cudaMemsetAsync(vis.p, 0, 8, s));
            ga.visits = vis.p;
          }
          static const int tq_sleep_max = getenv("BF_TQ_SLEEP_MAX") ? atoi(getenv("BF_TQ_SLEEP_MAX")) : 512;
          static const int tq_bigger_first = getenv("BF_TQ_BIGGER_FIRST") ? atoi(getenv("BF_TQ_BIGGER_FIRST")) : 1;
          ga.tq_sleep_max = tq_sleep_max < 32 ? 32 : tq_sleep_max;
          ga.tq_bigger_first = tq_bigger_first;
          static const int tq_lpt = getenv("BF_TQ_LPT") ? atoi(getenv("BF_TQ_LPT")) : 1;
          ga.tq_lpt = tq_lpt;
          static const bool want_stats = getenv("BF_SUBTREE_STATS") != nullptr;
          DBuf<unsigned long long> st;
          if (want_stats) {
            st.alloc(24, s);
            BF_CUDA_CHECK(cudaMemsetAsync(st.p, 0, 24 * 8, s));
            ga.stats = st.p;
          }
          {
            KScope ks_("k_subtree", s, 0.0);
            // helper warps (BF_SUBTREE_HW=4: 4 warps grow tiny nodes during the medium levels; ballot masks)
            static const int sub_hw = getenv("BF_SUBTREE_HW") ? atoi(getenv("BF_SUBTREE_HW")) : 0;
            if (tiny_v == 0)
              k_subtree<0, 64, 0><<<(unsigned)ngroups, SUB_NT, subtree_smem(A, p, 64), s>>>(ga);
            else if (sub_hw == 4 && tiny_max == 64)
              k_subtree<2, 64, 4><<<(unsigned)ngroups, SUB_NT, subtree_smem(A, p, 64), s>>>(ga);
            else if (sub_hw == 2 && tiny_max == 64)
              k_subtree<2, 64, 2><<<(unsigned)ngroups, SUB_NT, subtree_smem(A, p, 64), s>>>(ga);
            else if (tiny_v == 2)
              k_subtree<2, 64, 0><<<(unsigned)ngroups, SUB_NT, subtree_smem(A, p, 64), s>>>(ga);
            else if (tiny_v == 3 && tiny_max == 128)
              k_subtree<3, 128, 0><<<(unsigned)ngroups, SUB_NT, subtree_smem(A, p, 128), s>>>(ga);
            else if (tiny_v == 3)
              k_subtree<3, 64, 0><<<(unsigned)ngroups, SUB_NT, subtree_smem(A, p, 64), s>>>(ga);
            else if (tiny_max == 64)
              k_subtree<1, 64, 0><<<(unsigned)ngroups, SUB_NT, subtree_smem(A, p, 64), s>>>(ga);
            else
              k_subtree<1, 128, 0><<<(unsigned)ngroups, SUB_NT, subtree_smem(A, p, 128), s>>>(ga);
          }
          if (ga.visits) {  // SURVEY 8(d) split-search bytes of the subtree nodes: 20 B per entry visit
            unsigned long long hv = 0;
            d2h(&hv, vis.p, 1, s);
            BF_CUDA_CHECK(cudaStreamSynchronize(s));
            prof_add_bytes("k_subtree:scan_bytes", (double)hv * 20.0);
          }
          if (want_stats) {
            unsigned long long h[24];
            d2h(h, st.p, 24, s);
            BF_CUDA_CHECK(cudaStreamSynchronize(s));
            const double c = (double)h[5];
            fprintf(stderr, "[subtree tiny] draw=%.0f groups=%.0f per tiny node\n", h[11] / (double)(h[7] ? h[7] : 1), h[12] / (double)(h[7] ? h[7] : 1));
            fprintf(stderr, "[subtree tiny group] per tiny node: stage=%.0f passA=%.0f segscan=%.0f passB=%.0f wmax=%.0f passC=%.0f\n", h[21] / (double)(h[7] ? h[7] : 1), h[16] / (double)(h[7] ? h[7] : 1), h[17] / (double)(h[7] ? h[7] : 1), h[18] / (double)(h[7] ? h[7] : 1), h[19] / (double)(h[7] ? h[7] : 1), h[20] / (double)(h[7] ? h[7] : 1));
            fprintf(stderr, "[subtree medium] per cta: scan+finalize=%.0f (finalize %.0f) next=%.0f partition=%.0f cycles, %.2f levels\n", h[13] / (double)(h[5] ? h[5] : 1), h[23] / (double)(h[5] ? h[5] : 1), h[14] / (double)(h[5] ? h[5] : 1), h[15] / (double)(h[5] ? h[5] : 1), h[22] / (double)(h[5] ? h[5] : 1));
            fprintf(stderr, "[subtree] A=%d ctas=%llu mean_a0=%.1f cyc/cta: load=%.0f medium=%.0f tiny=%.0f flush=%.0f | medium nodes/cta=%.1f tiny nodes/cta=%.1f nodes/cta=%.1f warp-cyc in tiny/cta=%.0f busy=%.0f (%.0f per tiny node)\n",
                    A, h[5], h[6] / c, h[0] / c, h[1] / c, h[2] / c, h[3] / c, h[4] / c, h[7] / c, h[9] / c, h[8] / c,
                    h[10] / c, h[10] / (double)(h[7] ? h[7] : 1));
          }
          BF_CUDA_CHECK(cudaGetLastError());
        }
      }
      ptm.mark("subtree");
      // ---- a11 emit
      std::vector<int32_t> hnn(Bc);
      d2h(hnn.data(), pnn.p, Bc, s);
      BF_CUDA_CHECK(cudaStreamSynchronize(s));
      std::vector<int64_t> hoff(Bc);
      int64_t tot = 0;
      int32_t mx = 0;
      for (int b = 0; b < Bc; ++b) {
        hoff[b] = tot;
        tot += hnn[b];
        mx = std::max(mx, hnn[b]);
        F->tree_off[(size_t)(tb - prm.tree_begin + b) + 1] = hnn[b];
      }
      Chunk ch;
      ch.total = tot;
      ch.nodes.alloc(tot, s);
      ch.count.alloc(tot, s);
      ch.value.alloc(tot, s);
      ch.drss.alloc(tot, s);
      h2d(emit_off.p, hoff.data(), Bc, s);
      {
        KScope ks_("k_emit", s, 0.0);
        k_emit<<<dim3((unsigned)ceil_div(mx, NT), Bc), NT, 0, s>>>(pool, emit_off.p, ch.nodes.p, ch.count.p,
                                                                  ch.value.p, ch.drss.p);
      }
      BF_CUDA_CHECK(cudaGetLastError());
      chunks.push_back(std::move(ch));
    }
    // ---- assemble the forest
    for (int32_t i = 0; i < T_loc; ++i) F->tree_off[i + 1] += F->tree_off[i];
    const int64_t total = F->tree_off[T_loc];
    forest_alloc(F, total, T_loc, s);
    h2d(F->d_tree_off, F->tree_off.data(), (size_t)T_loc + 1, s);
    int64_t o = 0;
    for (auto& ch : chunks) {
      if (ch.total) {
        BF_CUDA_CHECK(cudaMemcpyAsync(F->d_nodes + o, ch.nodes.p, ch.total * sizeof(Node16), cudaMemcpyDeviceToDevice, s));
        BF_CUDA_CHECK(cudaMemcpyAsync(F->d_count + o, ch.count.p, ch.total * 4, cudaMemcpyDeviceToDevice, s));
        BF_CUDA_CHECK(cudaMemcpyAsync(F->d_value + o, ch.value.p, ch.total * 8, cudaMemcpyDeviceToDevice, s));
        BF_CUDA_CHECK(cudaMemcpyAsync(F->d_drss + o, ch.drss.p, ch.total * 8, cudaMemcpyDeviceToDevice, s));
      }
      o += ch.total;
    }
    chunks.clear();
    BF_CUDA_CHECK(cudaStreamSynchronize(s));
    ptm.mark("emit+assemble");
  } catch (...) {
    forest_release(F);
    delete F;
    throw;
  }
  *out = F;
}

}  // namespace bf
