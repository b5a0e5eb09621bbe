/*
 * bf.h -- C ABI of the B200-native BlackForest random-forest hot path.
 *
 * The method (PAPER.md = /root/reference/PAPER.md, "P:n" = line n):
 *   learning set (X, Y): N observations x p predictors, numeric response   P:71  (sec 4.1.1)
 *   regression tree = recursive binary partition, leaf = region mean       P:73-79, eq.(1)
 *   split on half-planes x_j <= s minimising RSS_L + RSS_R                 P:81-91, eqs.(2),(3)
 *   grow until a minimum node size (e.g. 5), no pruning in a forest
 *   forest: n_t bootstrap samples, random predictor subset per node,
 *           prediction = average of the trees
 *   permutation importance on OOB samples, tree by tree
 *   OOB error / variance explained
 *   PCA of the counters (prcomp)
 * The exact arithmetic, RNG streams and readings of silent passages are
 * DESIGN.md sections 2 (S1..S9) and 3 (R1..R20).
 *
 * Conventions
 *   - Matrices are COLUMN-MAJOR: element (i, j) at X[j*ld + i], ld >= rows.
 *   - Pointers may be CUDA device pointers or host pointers (pageable or
 *     pinned); the library detects host pointers with
 *     cudaPointerGetAttributes and stages them through device memory on the
 *     given stream (host<->device copies are then part of the call).
 *   - The caller owns every input and output buffer; the library never frees
 *     them.  The library owns bf_forest and its device memory (allocated
 *     through the bf_set_allocator hooks -- the Python binding installs the
 *     torch caching allocator -- else cudaMallocAsync on the call's stream).
 *   - Return value: BF_OK (0) or a negative BF_E* code; no exception crosses
 *     the ABI; on error outputs are unspecified and no forest is returned.
 *     bf_last_error() returns a thread-local message for the last failure.
 *   - bf_fit is synchronous (node counts are needed on the host).  Every other
 *     call enqueues on `stream` (a cudaStream_t, NULL = legacy default stream)
 *     and returns; results are valid after the stream is synchronised.  Calls
 *     that were given HOST output pointers synchronise before returning.
 */
#ifndef BF_H
#define BF_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define BF_ABI_VERSION 1

enum {
  BF_OK = 0,
  BF_EINVAL = -1,      /* bad shape, ld < rows, mtry not in [1,p], nodesize < 1, ntree < 1, bad tree range */
  BF_ENONFINITE = -2,  /* NaN/Inf in X or y (reading R17)                                                 */
  BF_ERANGE = -3,      /* n >= 2^31 or sampsize >= 2^31, or |y| range not representable                   */
  BF_ENOMEM = -4,      /* device allocation failed                                                        */
  BF_ECUDA = -5,       /* CUDA runtime error (message in bf_last_error)                                   */
  BF_ENOTIMPL = -6     /* e.g. replace = 0 with sampsize != n (reading R20)                               */
};

/* Forest parameters.  Defaults in brackets are the R randomForest regression
 * defaults the paper used (readings R3, R6).                          */
typedef struct bf_params {
  int32_t ntree;           /* T, total forest size [500]; global tree ids 0..T-1               */
  int32_t mtry;            /* predictors drawn per node; 0 -> max(floor(p/3), 1)               */
  int32_t nodesize;        /* a node with n_k <= nodesize is a leaf [5]                        */
  int32_t replace;         /* 1 bootstrap with replacement [1]; 0 every row once (sampsize==n) */
  int64_t sampsize;        /* N_s; 0 -> n                                                      */
  uint64_t seed;           /* Philox key (S1)                                                  */
  int32_t tree_begin;      /* this call grows global trees [tree_begin, tree_end)              */
  int32_t tree_end;        /*   (multi-GPU: each rank a disjoint range, possibly empty when
                              ntree < ranks; tree_end < 0 -> [0, ntree); begin == end -> an
                              empty forest, which predict / importance accept)               */
  int32_t trees_in_flight; /* trees grown concurrently; 0 -> auto from free device memory      */
  int32_t small_node_max;  /* largest node (distinct rows) grown by one CTA in shared memory;
                              0 -> auto from the shared-memory budget and p                    */
} bf_params;

typedef struct bf_forest bf_forest; /* opaque, library-owned, device-resident */

/* Summary of a forest (host struct filled by bf_forest_info). */
typedef struct bf_forest_info {
  int64_t n;              /* training rows                                */
  int32_t p;              /* predictors                                   */
  int32_t ntree_total;    /* T of the whole forest                        */
  int32_t tree_begin;     /* global id of the first tree held             */
  int32_t tree_end;       /* one past the last                            */
  int64_t total_nodes;    /* nodes over the held trees                    */
  int32_t q;              /* fixed-point exponent of S2                   */
  int32_t mtry, nodesize, replace;
  int64_t sampsize;
  uint64_t seed;
} bf_forest_info;

/* Flat view of a forest, used by export (host arrays written by the library)
 * and import (host or device arrays read by the library).  Nodes of local
 * tree i are [tree_off[i], tree_off[i+1]); node ids inside a tree are local
 * (root = 0; right child = left + 1).  feature = -1 marks a leaf.
 * thr_or_value = threshold for internal nodes, leaf value for leaves.       */
typedef struct bf_forest_view {
  bf_forest_info info;
  int64_t* tree_off;      /* ntrees + 1                                   */
  int32_t* feature;       /* total_nodes                                  */
  int32_t* left;          /* total_nodes                                  */
  double* thr_or_value;   /* total_nodes                                  */
  int32_t* count;         /* total_nodes: n_k (bootstrap duplicates counted) */
  double* value;          /* total_nodes: node mean (every node, eq.(1))  */
  double* drss;           /* total_nodes: RSS decrease of the split (S4.6), 0 for leaves */
} bf_forest_view;

/* OOB / importance accumulators for the trees of ONE forest object
 * (device pointers, caller-allocated; T_loc = tree_end - tree_begin).
 * Slots are per LOCAL tree so that ranks holding disjoint tree ranges can be
 * merged exactly by placing them at their global offsets (sum of disjoint
 * slots = all-gather).  bf_oob_importance overwrites all of them.           */
typedef struct bf_oob_accum {
  double* d_slots;        /* T_loc * p : d_tm (S7), row-major [tree][m]    */
  double* npur_slots;     /* T_loc * p : sum of drss of splits on m (S8)   */
  double* oob_sum;        /* n : sum of OOB tree predictions of row i (S6) */
  int32_t* oob_cnt;       /* n : number of OOB trees of row i              */
  double* e_t;            /* T_loc : OOB squared error of tree t           */
  int64_t* nout_t;        /* T_loc : OOB rows of tree t                    */
} bf_oob_accum;

/* ---------------------------------------------------------------------- */
const char* bf_version(void);
const char* bf_last_error(void);

/* Allocator hook for every device buffer the library owns (fit work space,
 * forests, staging copies of host inputs).  alloc(bytes, stream, ctx) returns
 * a block usable in `stream` order (NULL -> BF_ENOMEM); free(ptr, stream,
 * ctx) returns it in the order of the stream it was allocated on.  A forest
 * used on another stream is released only after cudaDeviceSynchronize.  The
 * Python binding installs torch's CUDA caching allocator (libbf_torch_alloc.so:
 * raw_alloc_with_stream / raw_delete), so the library and the caller's
 * tensors share one pool.  NULL hooks restore cudaMallocAsync /
 * cudaFreeAsync on the device's default memory pool.  Not thread-safe against
 * calls in flight: set it before the first call.                           */
typedef void* (*bf_alloc_fn)(size_t bytes, void* stream, void* ctx);
typedef void (*bf_free_fn)(void* ptr, void* stream, void* ctx);
int bf_set_allocator(bf_alloc_fn alloc, bf_free_fn free_, void* ctx);
/* Free device memory the caller's allocator can still hand out (bytes; 0 =
 * ask the driver with cudaMemGetInfo).  bf_fit sizes its trees in flight from
 * half of it.  The Python binding passes the driver's free memory plus the
 * torch caching allocator's cached-but-unused blocks before every fit.
 * BF_EINVAL for a negative value.                                          */
int bf_set_memory_budget(int64_t bytes);
/* Release the node-list work space bf_fit keeps across calls (the three list
 * buffers of the largest fit so far, reused by the next fits of that size;
 * BF_LIST_WORKSPACE=0 makes bf_fit allocate them per call instead).  Waits for
 * the device first.  BF_OK, or BF_EINVAL while a fit is using it.           */
int bf_release_workspace(void);

/* Grow global trees [tree_begin, tree_end) of a T-tree forest (P:95 steps 1-2;
 * S2-S4).  X: n x p column-major (ldx >= n), y: n.  Synchronous.  *out
 * receives a new forest owned by the caller (free with bf_forest_free).     */
int bf_fit(const double* X, int64_t ldx, const double* y, int64_t n, int32_t p,
           const bf_params* prm, void* stream, bf_forest** out);

void bf_forest_free(bf_forest* f);
int bf_forest_info_get(const bf_forest* f, bf_forest_info* info);
/* Export to HOST arrays sized from bf_forest_info (tree_off: ntrees + 1).  */
int bf_forest_export(const bf_forest* f, bf_forest_view* v);
/* Build a forest from a view (host or device arrays; used after the
 * multi-GPU gather).  info.tree_begin/tree_end give the held range.        */
int bf_forest_import(const bf_forest_view* v, void* stream, bf_forest** out);

/* Batched prediction (P:95 step 3; S5).  Xq: m x p column-major (ldq >= m).
 * yhat_sum[i] = sum over the forest's trees of the leaf value (may be NULL);
 * yhat[i] = yhat_sum[i] / ntree_total (may be NULL; ntree_total <= 0 ->
 * number of held trees).                                                   */
int bf_predict(const bf_forest* f, const double* Xq, int64_t ldq, int64_t m,
               double* yhat_sum, double* yhat, int32_t ntree_total, void* stream);

/* Partial dependence of the response on predictor m ("the partial
 * dependence plot, shows how the response changes as a predictor ...
 * change(s)"; readings R23, R24).  X: the n x p rows to
 * average over (column-major, ldx >= n; normally the training data), grid:
 * G values v_g of predictor m (host or device).
 *   pd_sum[g] = sum_i sum_{held t} f_t(x_i with x_im := v_g)   (may be NULL)
 *   pd[g]     = pd_sum[g] / (n * ntree_total)                  (may be NULL;
 *               ntree_total <= 0 -> number of held trees)
 * Multi-GPU: ranks holding disjoint tree ranges all-reduce pd_sum.         */
int bf_partial_dependence(const bf_forest* f, const double* X, int64_t ldx, int64_t n, int32_t p, int32_t m,
                          const double* grid, int32_t G, double* pd_sum, double* pd, int32_t ntree_total,
                          void* stream);
/* Default partial-dependence grid of a predictor column x (n values; reading
 * R23 = R randomForest partialPlot): G = min(n_pt, distinct values of x),
 * v_g = min + g * ((max - min) / (G - 1)) for g < G - 1, v_{G-1} = max
 * (G = 1: v_0 = min).  grid must hold n_pt values; *G (host) receives G.
 * Synchronous.                                                             */
int bf_pd_grid(const double* x, int64_t n, int32_t n_pt, double* grid, int32_t* G, void* stream);

/* OOB prediction + permutation importance over the forest's trees (P:130,
 * P:157; S6-S8).  X, y must be the training data of bf_fit.               */
int bf_oob_importance(const bf_forest* f, const double* X, int64_t ldx, const double* y,
                      int64_t n, int32_t p, const bf_oob_accum* acc, void* stream);

/* Aggregate accumulators of ALL ntree trees (slots in global tree order,
 * e.g. after an all-reduce of disjoint slots; S6-S8).  Outputs p-vectors and
 * two scalars (device or host pointers).                                   */
int bf_importance_finalize(const double* d_slots, const double* npur_slots, const double* oob_sum,
                           const int32_t* oob_cnt, const double* y, int64_t n, int32_t p, int32_t ntree,
                           double* inc_mse, double* inc_mse_raw, double* inc_mse_sd,
                           double* inc_node_purity, double* oob_mse, double* rsq, void* stream);

/* PCA of the counters (S9).  X: n x p column-major.  scale != 0
 * standardises columns (zero-variance column -> BF_EINVAL).  Outputs: sdev
 * (p), rotation (p x p column-major, column j = component j), center (p,
 * may be NULL), scores (n x k column-major, may be NULL).                  */
int bf_pca(const double* X, int64_t ldx, int64_t n, int32_t p, int32_t scale, int32_t k,
           double* sdev, double* rotation, double* center, double* scores, void* stream);

/* Number of retained principal components (reading R15; "a small
 * number of principal components (less than 10)", "4 PCs ... more than
 * 97%"): the smallest k with sum_{j<k} sdev_j^2 >= frac * sum_j sdev_j^2,
 * clamped to [1, min(cap, p)].  sdev: p values in descending order (bf_pca
 * output; device or host).  *k: HOST int32.  Synchronous.  BF_EINVAL for p
 * outside [1, 1024], cap < 1 or frac outside (0, 1].                       */
int bf_pca_retained(const double* sdev, int32_t p, double frac, int32_t cap, int32_t* k, void* stream);

/* Varimax rotation of factor loadings ("the factor loadings of the
 * variable with relation to the retained principal components"; reading R25
 * = R stats::varimax).  L: p x k column-major (ldl >= p), e.g. rotation[:, :k]
 * scaled by sdev[:k].  normalize != 0: rows scaled to unit length before and
 * back after (a zero row -> BF_EINVAL).  Iterates T <- U V^T of
 * B = x^T (Z^3 - Z diag(colsum(Z^2))/p), Z = x T, until the sum of singular
 * values d grows by less than a factor (1 + eps) [R: eps = 1e-5], at most 1000
 * times.  Outputs: loadings (p x k, ld = p), rotmat (k x k), *iters (host,
 * may be NULL).  1 <= k <= 32; 2 p k + p doubles must fit shared memory.
 * Synchronous.                                                             */
int bf_varimax(const double* L, int64_t ldl, int32_t p, int32_t k, int32_t normalize, double eps, double* loadings,
               double* rotmat, int32_t* iters, void* stream);

/* Counter models ("(generalized) linear models
 * are sufficient", "generalized linear models ... residual
 * deviance"; reading R26 = R glm, default gaussian family, identity link):
 * least squares of each of the r response columns of Y (n x r, column-major,
 * ldy >= n; e.g. retained counters) on the shared design Z (n x k,
 * column-major, ldz >= n; built by the caller from problem/platform
 * characteristics, intercept column included by the caller).  Outputs: coef
 * (k x r, ld k), deviance (r, residual sum of squares; may be NULL),
 * null_deviance (r, sum of squares about the mean; may be NULL).  Solved by
 * column-scaled CholeskyQR2 in fp64.  1 <= k <= 32, 1 <= r <= 64, n >= k;
 * a rank-deficient design -> BF_EINVAL.  Synchronous.                      */
int bf_glm_gaussian(const double* Z, int64_t ldz, int64_t n, int32_t k, const double* Y, int64_t ldy, int32_t r,
                    double* coef, double* deviance, double* null_deviance, void* stream);
/* The counter models on new rows ("generate values for the most
 * influential variables from an unseen problem size"): out (n x r,
 * column-major, ldo >= n) = Z (n x k, ldz >= n) coef (k x r, ld k).         */
int bf_glm_predict(const double* Z, int64_t ldz, int64_t n, int32_t k, const double* coef, int32_t r, double* out,
                   int64_t ldo, void* stream);
/* MARS counter models (eq. (4), P:173, P:256 R earth; reading R28:
 * earth's additive defaults).  X: n x d column-major predictors (ldx >= n;
 * problem / platform characteristics), y: n responses (one counter); host or
 * device.  Forward pass: hinge pairs max(0, x_v - t), max(0, t - x_v) at the
 * knots t = distinct values of x_v other than its min and max, the pair
 * giving the smallest RSS added each step (ties within 1e-12 TSS -> lowest v,
 * t) while the RSq gain >= thresh [0.001], RSq < 1 - thresh and terms + 2 <=
 * nk [0 -> min(200, max(20, 2 d)) + 1]; backward pass: greedy removal of the
 * term whose loss raises RSS least, subset with the smallest GCV =
 * (RSS/n) / (1 - C/n)^2, C = terms + penalty (terms - 1) / 2 [penalty 2].
 * Outputs (HOST): *nterms, term_var / term_knot / term_dir (0 = intercept,
 * +1 = max(0, x - t), -1 = max(0, t - x)) and coef, each >= nk long; stats =
 * {RSS, GCV, RSq}.  At most 31 terms.  Synchronous.                        */
int bf_mars_fit(const double* X, int64_t ldx, int64_t n, int32_t d, const double* y, int32_t nk, double thresh,
                double penalty, int32_t* nterms, int32_t* term_var, double* term_knot, int32_t* term_dir, double* coef,
                double* stats, void* stream);
/* A MARS model on new rows: out[i] = sum_j coef_j B_j(x_i).  Terms and coef
 * host or device; X (m x d, ldx >= m) and out host or device.              */
int bf_mars_predict(const double* X, int64_t ldx, int64_t m, int32_t d, int32_t nterms, const int32_t* term_var,
                    const double* term_knot, const int32_t* term_dir, const double* coef, double* out, void* stream);
/* Similarity of two importance rankings of the same p predictors (SURVEY 8(f)
 * NEXT-4; "the same variable importance ranking", P:295 platform
 * "similarity"; reading R27): out[0] = Spearman's rho (Pearson correlation of
 * mid-ranks), out[1] = Kendall's tau-b (ties excluded pairwise); NaN when a
 * vector is constant.  a, b, out: host or device.  2 p doubles must fit in
 * shared memory (p <= 14000).                                              */
int bf_rank_similarity(const double* a, const double* b, int32_t p, double* out, void* stream);

/* Default counter-model design of one problem characteristic (reading R26;
 * P:222 sizes 2^5..2^11, P:254 lengths 64..8192): u = (log2 s - mean) / sd
 * over the n sizes (sample sd, n - 1); Z row r at Z[r * ldz + i] (the k x n
 * design layout of bf_glm_gaussian) = [1, u, u^2, u^3].  size > 0; n >= 2.
 * Device or host pointers.                                                 */
int bf_log_size_design(const double* size, int64_t n, double* Z, int64_t ldz, void* stream);

/* Test error of predicted times ("variance explained"): out[0] = mse =
 * mean (yhat - y)^2, out[1] = 1 - mse / mean (y - mean y)^2 (NaN for constant
 * y).  out: HOST, 2 doubles.  Synchronous.                                 */
int bf_prediction_error(const double* yhat, const double* y, int64_t m, double* out, void* stream);

/* ---- single-step entry points (parity tests) ---- */
/* The hand-written device primitives under the presort (row a3)
 * and the per-level offsets: an ascending, stable LSD radix sort of nseg
 * independent segments of n 64-bit keys (keys[seg*n + i]) carrying optional
 * 32-bit values (vals may be NULL), in place; an exclusive (inclusive != 0:
 * inclusive) prefix sum of n uint32; the distinct values of n sorted keys
 * (*count: device int32).  Device pointers only (BF_EINVAL otherwise).
 * Synchronous.                                                             */
int bf_sort_u64(uint64_t* keys, uint32_t* vals, int64_t n, int32_t nseg, void* stream);
int bf_scan_u32(const uint32_t* in, uint32_t* out, int64_t n, int32_t inclusive, void* stream);
int bf_unique_u64(const uint64_t* sorted, int64_t n, uint64_t* out, int32_t* count, void* stream);
/* Philox4x32-10 on `count` counters (S1): ctr[4*i..], out[4*i..].          */
int bf_philox(const uint32_t* ctr, uint32_t key0, uint32_t key1, uint32_t* out, int64_t count, void* stream);
/* Correctly rounded int128 -> double of (hi[i], lo[i]) (the key of S4.3). */
int bf_i128_to_double(const int64_t* hi, const uint64_t* lo, double* out, int64_t count, void* stream);
/* S2 fixed point: yq (n int64), *q (host int32).  Synchronous.             */
int bf_fixed_point(const double* y, int64_t n, int64_t sampsize, int64_t* yq, int32_t* q, void* stream);
/* S3 BOOT multiplicities of global trees [t0, t0+ntrees): w[(t-t0)*n + i]. */
int bf_bootstrap(uint64_t seed, int32_t t0, int32_t ntrees, int64_t n, int64_t sampsize, int32_t replace,
                 int32_t* w, void* stream);
/* S7 Feistel pi_tm(a) for a = 0..n_o-1 into out[n_o].                      */
int bf_perm(uint64_t seed, int32_t t, int32_t m, int64_t n_o, int64_t* out, void* stream);

/* ---- measurement hooks (bench.py) ---------------------------------------
 * When enabled, the library records a CUDA event pair on the launching stream
 * around every kernel launch it makes, grouped by kernel class, together with
 * the launch's ALGORITHMIC bytes.  bf_profile_read
 * synchronises those events, returns the accumulated totals and resets them.
 * bf_launch_count counts every kernel launch the library has made (CUB
 * primitives count once per call), whether or not profiling is enabled.    */
typedef struct bf_kernel_stat {
  char name[40];
  double ms;         /* summed device time between the event pairs          */
  int64_t launches;  /* launches of this class                              */
  double bytes;      /* summed algorithmic bytes                            */
} bf_kernel_stat;
int bf_profile_enable(int on);
int bf_profile_read(bf_kernel_stat* stats, int cap, int* count);
int64_t bf_launch_count(void);

#ifdef __cplusplus
}
#endif
#endif /* BF_H */
