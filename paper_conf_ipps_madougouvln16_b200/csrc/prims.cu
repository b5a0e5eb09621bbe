// prims.cu -- hand-written device primitives for sm_100a used around the hot path:
// prefix scans (the per-level child/piece/item offsets of the fit, the presort's dense ranks), an LSD radix
// sort of 64-bit keys with optional 32-bit values (the per-feature presort of SURVEY 8(a) row a3, P:81-91:
// "the values x_j ... sorted"; the partial-dependence grid and the MARS knots), and unique of sorted keys.
//
// Scans: one CTA walks the array in tiles with a running carry when it is small (the per-level scans of a
// few thousand entries: one launch, no scratch); otherwise reduce -> scan of the tile sums -> scan of the
// tiles with their offsets (three launches, recursive on the tile sums).
// Radix sort: 8-bit digits, least significant first; a digit that is equal for every key (one pre-pass
// histogram of all eight digits) is skipped.  Per pass: per-tile digit counts, one exclusive scan of the
// digit-major count table, and a stable scatter: warp w of a tile ranks its 512 keys round by round with
// __match_any_sync (lanes holding the same digit), a per-warp running count per digit, then per-digit
// prefix sums over the warps.  Stability = tile order = warp order then round then lane.
#include <algorithm>

#include "bf_internal.cuh"

namespace bf {
namespace {

constexpr int SC_NT = 256;              // threads of a scan CTA
constexpr int SC_V = 8;                 // items per thread
constexpr int SC_TILE = SC_NT * SC_V;   // 2048 items per tile
constexpr int SC_SMALL = 1 << 13;       // up to this many items: one CTA

// Exclusive scan of one tile held blocked in registers (thread t: items t*V .. t*V+V-1).  Returns the tile
// total; v[] becomes exclusive (plus `carry`).
template <class T>
__device__ __forceinline__ T tile_scan(T (&v)[SC_V], T carry, T* wsum) {
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  T t = 0;
#pragma unroll
  for (int q = 0; q < SC_V; ++q) t += v[q];
  T inc = t;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const T u = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += u;
  }
  if (lane == 31) wsum[wid] = inc;
  __syncthreads();
  T wpre = 0, tot = 0;
#pragma unroll
  for (int k = 0; k < SC_NT / 32; ++k) {
    const T x = wsum[k];
    if (k < wid) wpre += x;
    tot += x;
  }
  __syncthreads();  // wsum reusable
  T run = carry + wpre + inc - t;
#pragma unroll
  for (int q = 0; q < SC_V; ++q) {
    const T x = v[q];
    v[q] = run;
    run += x;
  }
  return tot;
}

template <class T, bool INCL>
__global__ void __launch_bounds__(SC_NT) k_scan_small(const T* __restrict__ in, T* __restrict__ out, int64_t n) {
  __shared__ T wsum[SC_NT / 32];
  T carry = 0;
  for (int64_t b = 0; b < n; b += SC_TILE) {
    T v[SC_V];
    const int64_t j0 = b + (int64_t)threadIdx.x * SC_V;
#pragma unroll
    for (int q = 0; q < SC_V; ++q) v[q] = j0 + q < n ? in[j0 + q] : T(0);
    T keep[SC_V];
#pragma unroll
    for (int q = 0; q < SC_V; ++q) keep[q] = v[q];
    carry += tile_scan(v, carry, wsum);
#pragma unroll
    for (int q = 0; q < SC_V; ++q)
      if (j0 + q < n) out[j0 + q] = INCL ? v[q] + keep[q] : v[q];
  }
}

template <class T>
__global__ void __launch_bounds__(SC_NT) k_scan_reduce(const T* __restrict__ in, int64_t n, T* __restrict__ part) {
  __shared__ T wsum[SC_NT / 32];
  const int64_t j0 = (int64_t)blockIdx.x * SC_TILE + (int64_t)threadIdx.x * SC_V;
  T t = 0;
#pragma unroll
  for (int q = 0; q < SC_V; ++q) t += j0 + q < n ? in[j0 + q] : T(0);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) t += __shfl_down_sync(0xffffffffu, t, o);
  if (lane == 0) wsum[wid] = t;
  __syncthreads();
  if (threadIdx.x == 0) {
    T s = 0;
    for (int k = 0; k < SC_NT / 32; ++k) s += wsum[k];
    part[blockIdx.x] = s;
  }
}

template <class T, bool INCL>
__global__ void __launch_bounds__(SC_NT) k_scan_tiles(const T* __restrict__ in, T* __restrict__ out, int64_t n,
                                                      const T* __restrict__ part_excl) {
  __shared__ T wsum[SC_NT / 32];
  const int64_t j0 = (int64_t)blockIdx.x * SC_TILE + (int64_t)threadIdx.x * SC_V;
  T v[SC_V], keep[SC_V];
#pragma unroll
  for (int q = 0; q < SC_V; ++q) keep[q] = v[q] = j0 + q < n ? in[j0 + q] : T(0);
  tile_scan(v, part_excl[blockIdx.x], wsum);
#pragma unroll
  for (int q = 0; q < SC_V; ++q)
    if (j0 + q < n) out[j0 + q] = INCL ? v[q] + keep[q] : v[q];
}

template <class T, bool INCL>
void scan_impl(const T* in, T* out, int64_t n, cudaStream_t s) {
  if (n <= 0) return;
  if (n <= SC_SMALL) {
    KScope ks_("k_scan_small", s, 0.0);
    k_scan_small<T, INCL><<<1, SC_NT, 0, s>>>(in, out, n);
    BF_CUDA_CHECK(cudaGetLastError());
    return;
  }
  const int64_t nb = ceil_div(n, SC_TILE);
  DBuf<T> part(nb, s), pex(nb, s);
  {
    KScope ks_("k_scan_reduce", s, 0.0);
    k_scan_reduce<T><<<(unsigned)nb, SC_NT, 0, s>>>(in, n, part.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  scan_impl<T, false>(part.p, pex.p, nb, s);
  {
    KScope ks_("k_scan_tiles", s, 0.0);
    k_scan_tiles<T, INCL><<<(unsigned)nb, SC_NT, 0, s>>>(in, out, n, pex.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
}

// ------------------------------------------------------------------ LSD radix sort
constexpr int RS_NT = 256;
constexpr int RS_W = RS_NT / 32;        // warps per tile
constexpr int RS_R = 16;                // rounds of 32 keys per warp
constexpr int RS_TILE = RS_NT * RS_R;   // 4096 keys per tile
constexpr int RS_B = 256;               // 8-bit digits

// Histograms of all eight digits over every key (one pass; digits equal for every key are skipped).
__global__ void __launch_bounds__(RS_NT) k_rs_hist_all(const uint64_t* __restrict__ keys, int64_t n,
                                                       unsigned long long* __restrict__ hist /* 8 x 256 */) {
  __shared__ uint32_t h[8 * RS_B];
  for (int k = threadIdx.x; k < 8 * RS_B; k += RS_NT) h[k] = 0;
  __syncthreads();
  for (int64_t i = blockIdx.x * (int64_t)RS_NT + threadIdx.x; i < n; i += (int64_t)gridDim.x * RS_NT) {
    const uint64_t k = keys[i];
#pragma unroll
    for (int d = 0; d < 8; ++d) atomicAdd(&h[d * RS_B + (uint32_t)((k >> (8 * d)) & 0xff)], 1u);
  }
  __syncthreads();
  for (int k = threadIdx.x; k < 8 * RS_B; k += RS_NT)
    if (h[k]) atomicAdd(&hist[k], (unsigned long long)h[k]);
}

// Per-tile digit counts of segment blockIdx.y, digit-major within the segment: cnt[(seg * 256 + d) * nb + tile].
// An exclusive scan of the whole table then gives every (segment, digit, tile) its position in the
// concatenated output (segments are equal-length and keep their order).
__global__ void __launch_bounds__(RS_NT) k_rs_count(const uint64_t* __restrict__ keys, int64_t n, int shift,
                                                    uint32_t* __restrict__ cnt, int nb) {
  __shared__ uint32_t h[RS_B];
  h[threadIdx.x] = 0;
  __syncthreads();
  const uint64_t* kseg = keys + (int64_t)blockIdx.y * n;
  const int64_t t0 = (int64_t)blockIdx.x * RS_TILE;
#pragma unroll 4
  for (int r = 0; r < RS_R; ++r) {
    const int64_t i = t0 + (int64_t)r * RS_NT + threadIdx.x;
    if (i < n) atomicAdd(&h[(uint32_t)(kseg[i] >> shift) & 0xff], 1u);
  }
  __syncthreads();
  cnt[((int64_t)blockIdx.y * RS_B + threadIdx.x) * nb + blockIdx.x] = h[threadIdx.x];
}

// Stable scatter of one tile.  Warp w owns tile keys [w*512, (w+1)*512), read in rounds of 32 (coalesced).
template <bool VALS>
__global__ void __launch_bounds__(RS_NT) k_rs_scatter(const uint64_t* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                      uint64_t* __restrict__ kout, uint32_t* __restrict__ vout,
                                                      int64_t n, int shift, const uint32_t* __restrict__ off, int nb) {
  __shared__ uint32_t wh[RS_W][RS_B];
  __shared__ uint32_t soff[RS_B];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  for (int k = tid; k < RS_W * RS_B; k += RS_NT) (&wh[0][0])[k] = 0;
  soff[tid] = off[((int64_t)blockIdx.y * RS_B + tid) * nb + blockIdx.x];
  __syncthreads();
  kin += (int64_t)blockIdx.y * n;
  if (VALS) vin += (int64_t)blockIdx.y * n;
  const int64_t base = (int64_t)blockIdx.x * RS_TILE + (int64_t)wid * (RS_R * 32);
  uint64_t key[RS_R];
  uint32_t val[RS_R];
  uint16_t loc[RS_R];
#pragma unroll
  for (int r = 0; r < RS_R; ++r) {
    const int64_t i = base + r * 32 + lane;
    key[r] = i < n ? kin[i] : 0ull;
    if (VALS) val[r] = i < n ? vin[i] : 0u;
  }
  const unsigned lt = (1u << lane) - 1u;
#pragma unroll
  for (int r = 0; r < RS_R; ++r) {
    const int64_t i = base + r * 32 + lane;
    const bool ok = i < n;
    const unsigned vm = __ballot_sync(0xffffffffu, ok);
    if (ok) {
      const uint32_t d = (uint32_t)(key[r] >> shift) & 0xff;
      const unsigned peers = __match_any_sync(vm, d);
      const int leader = __ffs(peers) - 1;
      uint32_t b = 0;
      if (lane == leader) {
        b = wh[wid][d];
        wh[wid][d] = b + __popc(peers);
      }
      b = __shfl_sync(vm, b, leader);
      loc[r] = (uint16_t)(b + __popc(peers & lt));
    }
    __syncwarp();
  }
  __syncthreads();
  {  // per digit: exclusive prefix over the warps
    uint32_t run = 0;
#pragma unroll
    for (int w = 0; w < RS_W; ++w) {
      const uint32_t c = wh[w][tid];
      wh[w][tid] = run;
      run += c;
    }
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < RS_R; ++r) {
    const int64_t i = base + r * 32 + lane;
    if (i < n) {
      const uint32_t d = (uint32_t)(key[r] >> shift) & 0xff;
      const int64_t dst = (int64_t)soff[d] + wh[wid][d] + loc[r];
      kout[dst] = key[r];
      if (VALS) vout[dst] = val[r];
    }
  }
}

__global__ void k_unique_flags(const uint64_t* __restrict__ k, int64_t n, uint32_t* __restrict__ fl) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n) fl[i] = (i == 0 || k[i] != k[i - 1]) ? 1u : 0u;
}
__global__ void k_unique_scatter(const uint64_t* __restrict__ k, int64_t n, const uint32_t* __restrict__ fl,
                                 const uint32_t* __restrict__ pos, uint64_t* __restrict__ out, int32_t* __restrict__ cnt) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n && fl[i]) out[pos[i]] = k[i];
  if (i == n - 1) *cnt = (int32_t)(pos[i] + fl[i]);
}

}  // namespace

void scan_exclusive(const uint64_t* in, uint64_t* out, int64_t n, cudaStream_t s) { scan_impl<uint64_t, false>(in, out, n, s); }
void scan_exclusive(const int32_t* in, int32_t* out, int64_t n, cudaStream_t s) { scan_impl<int32_t, false>(in, out, n, s); }
void scan_exclusive(const uint32_t* in, uint32_t* out, int64_t n, cudaStream_t s) { scan_impl<uint32_t, false>(in, out, n, s); }
void scan_inclusive(const uint32_t* in, uint32_t* out, int64_t n, cudaStream_t s) { scan_impl<uint32_t, true>(in, out, n, s); }

const uint64_t* radix_sort_u64(uint64_t* k0, uint64_t* k1, uint32_t* v0, uint32_t* v1, int64_t n, int nseg,
                               cudaStream_t s, uint32_t** vals_out) {
  if (vals_out) *vals_out = v0;
  if (n <= 1 || nseg < 1) return k0;
  BF_REQUIRE(n * nseg < (int64_t(1) << 32), BF_ENOTIMPL, "radix sort: more than 2^32 keys");
  const int64_t tot = n * nseg;
  DBuf<unsigned long long> hist(8 * RS_B, s);
  BF_CUDA_CHECK(cudaMemsetAsync(hist.p, 0, sizeof(unsigned long long) * 8 * RS_B, s));
  {
    KScope ks_("k_rs_hist_all", s, 0.0);
    k_rs_hist_all<<<(unsigned)std::min<int64_t>(ceil_div(tot, RS_NT), 1184), RS_NT, 0, s>>>(k0, tot, hist.p);
  }
  BF_CUDA_CHECK(cudaGetLastError());
  std::vector<unsigned long long> h(8 * RS_B);
  BF_CUDA_CHECK(cudaMemcpyAsync(h.data(), hist.p, sizeof(unsigned long long) * 8 * RS_B, cudaMemcpyDeviceToHost, s));
  BF_CUDA_CHECK(cudaStreamSynchronize(s));
  const int nb = (int)ceil_div(n, RS_TILE);
  DBuf<uint32_t> cnt((size_t)RS_B * nb * nseg, s), off((size_t)RS_B * nb * nseg, s);
  uint64_t *ki = k0, *ko = k1;
  uint32_t *vi = v0, *vo = v1;
  const dim3 grid((unsigned)nb, (unsigned)nseg);
  for (int d = 0; d < 8; ++d) {
    bool constant = false;  // the digit is the same for every key of every segment: the pass is the identity
    for (int b = 0; b < RS_B; ++b) constant |= h[d * RS_B + b] == (unsigned long long)tot;
    if (constant) continue;
    const int shift = 8 * d;
    {
      KScope ks_("k_rs_count", s, 0.0);
      k_rs_count<<<grid, RS_NT, 0, s>>>(ki, n, shift, cnt.p, nb);
    }
    scan_exclusive(cnt.p, off.p, (int64_t)RS_B * nb * nseg, s);
    {
      KScope ks_("k_rs_scatter", s, 0.0);
      if (vi)
        k_rs_scatter<true><<<grid, RS_NT, 0, s>>>(ki, vi, ko, vo, n, shift, off.p, nb);
      else
        k_rs_scatter<false><<<grid, RS_NT, 0, s>>>(ki, nullptr, ko, nullptr, n, shift, off.p, nb);
    }
    BF_CUDA_CHECK(cudaGetLastError());
    std::swap(ki, ko);
    std::swap(vi, vo);
  }
  if (vals_out) *vals_out = vi;
  return ki;
}

void unique_u64(const uint64_t* sorted, int64_t n, uint64_t* out, int32_t* count_dev, cudaStream_t s) {
  if (n <= 0) {
    BF_CUDA_CHECK(cudaMemsetAsync(count_dev, 0, sizeof(int32_t), s));
    return;
  }
  DBuf<uint32_t> fl(n, s), pos(n, s);
  {
    KScope ks_("k_unique_flags", s, 0.0);
    k_unique_flags<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>(sorted, n, fl.p);
  }
  scan_exclusive(fl.p, pos.p, n, s);
  {
    KScope ks_("k_unique_scatter", s, 0.0);
    k_unique_scatter<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>(sorted, n, fl.p, pos.p, out, count_dev);
  }
  BF_CUDA_CHECK(cudaGetLastError());
}

}  // namespace bf
