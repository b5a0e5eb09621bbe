/*
 * bfo.h -- CPU ORACLE for the BlackForest random-forest hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_ipps_madougouvln16_b200/) never links,
 * imports or executes anything under oracle/.  It shares no source, header,
 * table or helper with the CUDA path (include/bf.h, csrc/).
 *
 * What it computes (DESIGN.md section 2 "Method spec", S1..S9):
 *   PAPER.md:71  (sec 4.1.1)  learning set (X, Y), N obs x p predictors
 *   PAPER.md:75-79 eq.(1)     piecewise-constant tree, leaf value = region mean
 *   PAPER.md:81-84 eq.(2)     half-plane split x_j <= s
 *   PAPER.md:86-91 eq.(3)     split minimising RSS_L + RSS_R
 *   PAPER.md:93               stop at a minimum node size (e.g. 5)
 *   PAPER.md:95               bootstrap samples, random predictor subset per
 *                             node, unpruned trees, prediction = tree average
 *   PAPER.md:130              OOB permutation importance, tree by tree
 *   PAPER.md:157              OOB error / variance explained
 * Readings where the paper is silent are listed in DESIGN.md section 3.
 *
 * Matrices are column-major: X[j*ldx + i] is predictor j of observation i.
 * All pointers are HOST pointers.  Return 0 on success, negative on error.
 */
#ifndef BFO_H
#define BFO_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { BFO_OK = 0, BFO_EINVAL = -1, BFO_ENONFINITE = -2, BFO_ERANGE = -3,
       BFO_ENOMEM = -4, BFO_ENOTIMPL = -6 };

typedef struct bfo_params {
  int32_t ntree;       /* total forest size T (global tree ids 0..T-1)        */
  int32_t mtry;        /* 0 -> max(floor(p/3), 1)                             */
  int32_t nodesize;    /* nodes with n_k <= nodesize are leaves (default 5)   */
  int32_t replace;     /* 1: bootstrap with replacement; 0: every row once    */
  int64_t sampsize;    /* 0 -> n                                              */
  uint64_t seed;       /* Philox key                                          */
  int32_t tree_begin;  /* grow global trees [tree_begin, tree_end)            */
  int32_t tree_end;
  int32_t nthreads;    /* host threads, one tree per thread (0 -> 1)          */
  int32_t pad_;
} bfo_params;

typedef struct bfo_forest bfo_forest;

/* --- primitives exposed for pinning ------------------------------------ */
/* Philox4x32-10 (Salmon et al. SC'11): out[0..3] from ctr[0..3], key[0..1]. */
void bfo_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
/* floor(u * r / 2^64) */
uint64_t bfo_mulhi64(uint64_t u, uint64_t r);
/* Fixed-point response (spec S2): fills yq[n], returns q through *q.        */
int bfo_fixed_point(const double* y, int64_t n, int64_t sampsize, int64_t* yq, int32_t* q);
/* Bootstrap multiplicities of global tree t (spec S3 BOOT).                 */
int bfo_bootstrap(uint64_t seed, int32_t t, int64_t n, int64_t sampsize, int32_t replace, int32_t* w);
/* mtry draw for a node with key K (spec S3 MTRY), writes mtry features.     */
void bfo_draw_mtry(uint64_t seed, int32_t t, uint64_t key, int32_t p, int32_t mtry, int32_t* feats);
/* Child key (spec S3 KEY).                                                  */
uint64_t bfo_child_key(uint64_t seed, int32_t t, uint64_t key, int32_t side);
/* Feistel permutation pi_tm(a) on [0, n_o) (spec S7).                       */
int64_t bfo_perm(uint64_t seed, int32_t t, int32_t m, int64_t n_o, int64_t a);
/* Correctly rounded int128 -> double, input as (hi, lo) two's complement.   */
double bfo_i128_to_double(int64_t hi, uint64_t lo);

/* --- forest ------------------------------------------------------------- */
int  bfo_fit(const double* X, int64_t ldx, const double* y, int64_t n, int32_t p,
             const bfo_params* prm, bfo_forest** out);
void bfo_forest_free(bfo_forest* f);
int32_t bfo_forest_ntrees(const bfo_forest* f);          /* tree_end - tree_begin */
int32_t bfo_forest_q(const bfo_forest* f);
/* Number of nodes of local tree i (0-based within [tree_begin, tree_end)).  */
int64_t bfo_tree_nnodes(const bfo_forest* f, int32_t i);
/* Copy tree i in BFS order.  feature = -1 for a leaf; thr only for internal
 * nodes (0 for leaves); left = BFS id of the left child (right = left + 1),
 * -1 for leaves; count = n_k (bootstrap duplicates counted); value = node
 * mean RN(sum w*y / n_k); drss = decrease of RSS (spec S4) or 0.            */
int bfo_tree_export(const bfo_forest* f, int32_t i, int32_t* feature, double* thr, int32_t* left,
                    int64_t* count, double* value, double* drss);

/* yhat_sum[r] = sum over this forest's trees of leaf value (tree order).     */
int bfo_predict(const bfo_forest* f, const double* Xq, int64_t ldq, int64_t m, double* yhat_sum);

/* OOB + permutation importance (spec S6-S8), partial over this forest's
 * trees.  Slots are indexed by LOCAL tree i: d_slots[i*p + m] = d_tm,
 * npur_slots[i*p + m] = sum of drss of splits on m in tree i.
 * oob_sum[r], oob_cnt[r]: sum / count of OOB predictions of row r.
 * e_t[i]: OOB squared error of tree i, nout_t[i]: its OOB row count.
 * perm_identity != 0 replaces pi by the identity (test hook).               */
int bfo_oob_importance(const bfo_forest* f, const double* X, int64_t ldx, const double* y,
                       int64_t n, int32_t p, int32_t perm_identity,
                       double* d_slots, double* npur_slots, double* oob_sum, int32_t* oob_cnt,
                       double* e_t, int64_t* nout_t);

/* Aggregation over ALL T trees (slots for t = 0..T-1 in tree order).        */
int bfo_importance_finalize(const double* d_slots, const double* npur_slots, const double* oob_sum,
                            const int32_t* oob_cnt, const double* y, int64_t n, int32_t p, int32_t ntree,
                            double* inc_mse, double* inc_mse_raw, double* inc_mse_sd,
                            double* inc_node_purity, double* oob_mse, double* rsq);

#ifdef __cplusplus
}
#endif
#endif
