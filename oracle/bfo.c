/*
 * bfo.c -- CPU ORACLE for the BlackForest random-forest hot path.
 *
 * TEST INFRASTRUCTURE ONLY (see bfo.h).  Plain, slow, single-threaded per
 * tree, written for reading against the paper and DESIGN.md section 2.
 * Compile with -O2 -ffp-contract=off (no FMA contraction: every fp64 result
 * below is one correctly rounded IEEE operation).
 *
 * Every function cites the passage it follows:  P:n = /root/reference/PAPER.md
 * line n; S1..S9 = DESIGN.md section 2 (the method spec, incl. the readings of
 * section 3 where the paper is silent).
 */
#define _GNU_SOURCE
#include "bfo.h"

#include <float.h>
#include <math.h>
#include <pthread.h>
#include <stdlib.h>
#include <string.h>

typedef __int128 i128;
typedef unsigned __int128 u128;

/* ------------------------------------------------------------------------ */
/* S1  Philox4x32-10 (Salmon, Moraes, Dror, Shaw, SC'11; Random123).          */
/* ------------------------------------------------------------------------ */
void bfo_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  uint32_t c0 = ctr[0], c1 = ctr[1], c2 = ctr[2], c3 = ctr[3];
  uint32_t k0 = key[0], k1 = key[1];
  for (int r = 0; r < 10; r++) {
    uint64_t p0 = (uint64_t)0xD2511F53u * c0;
    uint64_t p1 = (uint64_t)0xCD9E8D57u * c2;
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c1 ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c3 ^ k1;
    uint32_t n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* Two 64-bit draws from one Philox call: U0 = x0 | x1<<32, U1 = x2 | x3<<32 (S1). */
static void philox_u64x2(uint64_t seed, uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                         uint64_t* u0, uint64_t* u1) {
  uint32_t ctr[4] = {c0, c1, c2, c3};
  uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
  uint32_t x[4];
  bfo_philox4x32_10(ctr, key, x);
  *u0 = (uint64_t)x[0] | ((uint64_t)x[1] << 32);
  *u1 = (uint64_t)x[2] | ((uint64_t)x[3] << 32);
}

uint64_t bfo_mulhi64(uint64_t u, uint64_t r) { return (uint64_t)(((u128)u * (u128)r) >> 64); }

double bfo_i128_to_double(int64_t hi, uint64_t lo) {
  i128 v = (i128)(((u128)(uint64_t)hi << 64) | (u128)lo);
  return (double)v; /* libgcc __floattidf: correctly rounded, nearest-even */
}

static int bitlen_u64(uint64_t v) {
  int b = 0;
  while (v) { b++; v >>= 1; }
  return b;
}

static double canon(double x) { return x + 0.0; } /* -0.0 -> +0.0 (reading R18) */

/* ------------------------------------------------------------------------ */
/* S2  Fixed-point response: exact integer sums for eq.(3).        */
/* ------------------------------------------------------------------------ */
int bfo_fixed_point(const double* y, int64_t n, int64_t sampsize, int64_t* yq, int32_t* q) {
  if (n < 1) return BFO_EINVAL;
  double ymin = y[0], ymax = y[0];
  for (int64_t i = 0; i < n; i++) {
    if (!isfinite(y[i])) return BFO_ENONFINITE;
    if (y[i] < ymin) ymin = y[i];
    if (y[i] > ymax) ymax = y[i];
  }
  double c = 0.5 * ymin + 0.5 * ymax;
  double R = 0.0;
  for (int64_t i = 0; i < n; i++) {
    double d = fabs(y[i] - c);
    if (d > R) R = d;
  }
  if (!isfinite(R)) return BFO_ERANGE;
  if (R == 0.0) {
    for (int64_t i = 0; i < n; i++) yq[i] = 0;
    *q = 0;
    return BFO_OK;
  }
  int e;
  frexp(R, &e); /* R in [2^(e-1), 2^e) */
  int s = bitlen_u64((uint64_t)sampsize);
  int qq = 62 - s - e;
  for (int64_t i = 0; i < n; i++) yq[i] = llrint(ldexp(y[i] - c, qq));
  *q = qq;
  return BFO_OK;
}

/* ------------------------------------------------------------------------ */
/* S3  Random streams.  BOOT: ctr (j>>1, t, 1, 0), draw U_{j&1}.              */
/*     bootstrap sample of P:95 step 1 ("compose n_t bootstrap samples").    */
/* ------------------------------------------------------------------------ */
int bfo_bootstrap(uint64_t seed, int32_t t, int64_t n, int64_t sampsize, int32_t replace, int32_t* w) {
  if (n < 1) return BFO_EINVAL;
  if (!replace) {
    if (sampsize != n) return BFO_ENOTIMPL;
    for (int64_t i = 0; i < n; i++) w[i] = 1;
    return BFO_OK;
  }
  for (int64_t i = 0; i < n; i++) w[i] = 0;
  for (int64_t j = 0; j < sampsize; j++) {
    uint64_t u0, u1;
    philox_u64x2(seed, (uint32_t)(j >> 1), (uint32_t)t, 1u, 0u, &u0, &u1);
    uint64_t u = (j & 1) ? u1 : u0;
    int64_t row = (int64_t)bfo_mulhi64(u, (uint64_t)n);
    w[row] += 1;
  }
  return BFO_OK;
}

/* KEY: child key = U0 of ctr (K_lo, K_hi, t, 0x40000000 | side); root key 0. */
uint64_t bfo_child_key(uint64_t seed, int32_t t, uint64_t key, int32_t side) {
  uint64_t u0, u1;
  philox_u64x2(seed, (uint32_t)key, (uint32_t)(key >> 32), (uint32_t)t, 0x40000000u | (uint32_t)side, &u0, &u1);
  return u0;
}

/* MTRY: partial Fisher-Yates over [0, p) ("choosing randomly at each node a
 * subset of predictors").  Draw i uses ctr (K_lo, K_hi, t,
 * 0x20000000 | (i>>1)), word U_{i&1}.                                       */
void bfo_draw_mtry(uint64_t seed, int32_t t, uint64_t key, int32_t p, int32_t mtry, int32_t* feats) {
  int32_t* mind = (int32_t*)malloc(sizeof(int32_t) * (size_t)p);
  for (int32_t j = 0; j < p; j++) mind[j] = j;
  int32_t last = p - 1;
  for (int32_t i = 0; i < mtry; i++) {
    uint64_t u0, u1;
    philox_u64x2(seed, (uint32_t)key, (uint32_t)(key >> 32), (uint32_t)t, 0x20000000u | (uint32_t)(i >> 1), &u0, &u1);
    uint64_t u = (i & 1) ? u1 : u0;
    int32_t j = (int32_t)bfo_mulhi64(u, (uint64_t)(last + 1));
    feats[i] = mind[j];
    int32_t tmp = mind[j];
    mind[j] = mind[last];
    mind[last] = tmp;
    last--;
  }
  free(mind);
}

/* ------------------------------------------------------------------------ */
/* S4  Tree growth.                                                 */
/* ------------------------------------------------------------------------ */
typedef struct {
  int32_t feature; /* -1 leaf */
  double thr;
  int32_t left;
  int64_t count;
  double value;
  double drss;
} onode;

typedef struct {
  onode* nodes;
  int64_t nnodes, cap;
} otree;

struct bfo_forest {
  int64_t n;
  int32_t p, ntree, tree_begin, tree_end, q, mtry, nodesize, replace;
  int64_t sampsize;
  uint64_t seed;
  otree* trees;
};

typedef struct {
  int64_t* rows; /* distinct in-bag rows, ascending */
  int64_t a;
  uint64_t key;
  int32_t id;    /* BFS id */
} qitem;

typedef struct {
  const double* X;   /* canonicalised copy, column-major, ld = n */
  const double* y;
  const int64_t* yq;
  const int32_t* w;
  int64_t n;
  int32_t p, mtry, nodesize, q, t;
  uint64_t seed;
} grow_ctx;

static int push_node(otree* tr) {
  if (tr->nnodes == tr->cap) {
    tr->cap = tr->cap ? tr->cap * 2 : 64;
    tr->nodes = (onode*)realloc(tr->nodes, sizeof(onode) * (size_t)tr->cap);
  }
  onode* nd = &tr->nodes[tr->nnodes];
  nd->feature = -1; nd->thr = 0.0; nd->left = -1; nd->count = 0; nd->value = 0.0; nd->drss = 0.0;
  return (int)tr->nnodes++;
}

/* sort helper: rows ordered by x_f, ties by row (any tie order is allowed). */
static __thread const double* t_sort_col;
static int cmp_by_x(const void* A, const void* B) {
  int64_t ra = *(const int64_t*)A, rb = *(const int64_t*)B;
  double xa = t_sort_col[ra], xb = t_sort_col[rb];
  if (xa < xb) return -1;
  if (xa > xb) return 1;
  return (ra > rb) - (ra < rb);
}

/* eq.(3) key of one candidate boundary, S4:
 *   D = n_k*S_l - n_l*S_k (exact int128);
 *   g = RN( RN( RN(D)*RN(D) ) / RN(n_l*n_r) ).
 * g/n_k = D^2/(n_k n_l n_r) = RSS(parent) - RSS_L - RSS_R on y_q.          */
static double split_key(int64_t nk, int64_t Sk, int64_t nl, int64_t Sl) {
  i128 D = (i128)nk * (i128)Sl - (i128)nl * (i128)Sk;
  double d = (double)D;
  double nn = (double)(nl * (nk - nl));
  return (d * d) / nn;
}

static void grow_tree(const grow_ctx* c, otree* tr) {
  const int64_t n = c->n;
  int32_t p = c->p;
  /* root: every row with w > 0, ascending (P:95 bootstrap sample) */
  int64_t a0 = 0;
  for (int64_t i = 0; i < n; i++) a0 += (c->w[i] > 0);
  int64_t qcap = 64, qhead = 0, qtail = 0;
  qitem* queue = (qitem*)malloc(sizeof(qitem) * (size_t)qcap);
  qitem root;
  root.rows = (int64_t*)malloc(sizeof(int64_t) * (size_t)(a0 ? a0 : 1));
  root.a = 0;
  for (int64_t i = 0; i < n; i++)
    if (c->w[i] > 0) root.rows[root.a++] = i;
  root.key = 0;
  root.id = push_node(tr);
  queue[qtail++] = root;

  int32_t* feats = (int32_t*)malloc(sizeof(int32_t) * (size_t)(c->mtry > 0 ? c->mtry : 1));
  int64_t* srt = (int64_t*)malloc(sizeof(int64_t) * (size_t)(a0 ? a0 : 1));

  while (qhead < qtail) {
    qitem it = queue[qhead++];
    onode* nd = &tr->nodes[it.id];
    /* n_k, S_k, node value (eq.(1): c_m = mean of y in R_m), ascending rows */
    int64_t nk = 0, Sk = 0;
    double sy = 0.0;
    for (int64_t j = 0; j < it.a; j++) {
      int64_t r = it.rows[j];
      nk += c->w[r];
      Sk += (int64_t)c->w[r] * c->yq[r];
      sy += (double)c->w[r] * c->y[r];
    }
    nd->count = nk;
    nd->value = sy / (double)nk;
    /* P:93 stop at minimum node size: n_k <= nodesize -> leaf */
    if (nk <= c->nodesize) { free(it.rows); continue; }

    bfo_draw_mtry(c->seed, c->t, it.key, p, c->mtry, feats);

    int have = 0;
    double bg = 0.0;
    int32_t bf = -1;
    double ba = 0.0, bb = 0.0; /* values on each side of the best boundary */
    for (int32_t s = 0; s < c->mtry; s++) {
      int32_t f = feats[s];
      const double* col = c->X + (int64_t)f * n;
      memcpy(srt, it.rows, sizeof(int64_t) * (size_t)it.a);
      t_sort_col = col;
      qsort(srt, (size_t)it.a, sizeof(int64_t), cmp_by_x);
      int64_t nl = 0, Sl = 0;
      for (int64_t j = 0; j + 1 < it.a; j++) {
        int64_t r = srt[j];
        nl += c->w[r];
        Sl += (int64_t)c->w[r] * c->yq[r];
        double xa = col[r], xb = col[srt[j + 1]];
        if (!(xa < xb)) continue; /* not a boundary between distinct values */
        double g = split_key(nk, Sk, nl, Sl);
        /* best = max of (g, -f, -boundary); boundaries of one f are visited
         * in increasing order, features in any order -> explicit compare  */
        int better;
        if (!have) better = 1;
        else if (g > bg) better = 1;
        else if (g < bg) better = 0;
        else if (f < bf) better = 1;
        else if (f > bf) better = 0;
        else better = (xa < ba);
        if (better) { have = 1; bg = g; bf = f; ba = xa; bb = xb; }
      }
    }
    if (!have || bg == 0.0) { free(it.rows); continue; } /* no positive decrease -> leaf */

    /* split (eq.(2)): threshold inside the gap (a, b), reading R2 */
    double thr = 0.5 * ba + 0.5 * bb;
    if (!(thr < bb)) thr = ba;
    if (thr < ba) thr = ba;
    nd->feature = bf;
    nd->thr = thr;
    nd->drss = ldexp(bg / (double)nk, -2 * c->q);
    int32_t lid = push_node(tr);
    int32_t rid = push_node(tr);
    nd = &tr->nodes[it.id]; /* realloc may have moved it */
    nd->left = lid;

    const double* col = c->X + (int64_t)bf * n;
    qitem L, R;
    L.rows = (int64_t*)malloc(sizeof(int64_t) * (size_t)it.a);
    R.rows = (int64_t*)malloc(sizeof(int64_t) * (size_t)it.a);
    L.a = R.a = 0;
    for (int64_t j = 0; j < it.a; j++) {
      int64_t r = it.rows[j];
      if (col[r] <= thr) L.rows[L.a++] = r;
      else R.rows[R.a++] = r;
    }
    L.key = bfo_child_key(c->seed, c->t, it.key, 0);
    R.key = bfo_child_key(c->seed, c->t, it.key, 1);
    L.id = lid;
    R.id = rid;
    free(it.rows);
    if (qtail + 2 > qcap) {
      /* compact the consumed prefix, then grow */
      memmove(queue, queue + qhead, sizeof(qitem) * (size_t)(qtail - qhead));
      qtail -= qhead;
      qhead = 0;
      if (qtail + 2 > qcap) {
        qcap *= 2;
        queue = (qitem*)realloc(queue, sizeof(qitem) * (size_t)qcap);
      }
    }
    queue[qtail++] = L;
    queue[qtail++] = R;
  }
  free(queue);
  free(feats);
  free(srt);
}

/* ------------------------------------------------------------------------ */
/* bfo_fit: P:95 steps 1-2 for global trees [tree_begin, tree_end).           */
/* ------------------------------------------------------------------------ */
typedef struct {
  bfo_forest* F;
  const double* Xc;
  const double* y;
  const int64_t* yq;
  int next;            /* next local tree (guarded by mu) */
  pthread_mutex_t mu;
  int err;
} fit_job;

static void* fit_worker(void* arg) {
  fit_job* J = (fit_job*)arg;
  bfo_forest* F = J->F;
  int32_t* w = (int32_t*)malloc(sizeof(int32_t) * (size_t)F->n);
  for (;;) {
    pthread_mutex_lock(&J->mu);
    int i = J->next++;
    pthread_mutex_unlock(&J->mu);
    if (i >= F->tree_end - F->tree_begin) break;
    int32_t t = F->tree_begin + i;
    int rc = bfo_bootstrap(F->seed, t, F->n, F->sampsize, F->replace, w);
    if (rc) { J->err = rc; break; }
    grow_ctx c = {J->Xc, J->y, J->yq, w, F->n, F->p, F->mtry, F->nodesize, F->q, t, F->seed};
    grow_tree(&c, &F->trees[i]);
  }
  free(w);
  return NULL;
}

int bfo_fit(const double* X, int64_t ldx, const double* y, int64_t n, int32_t p,
            const bfo_params* prm, bfo_forest** out) {
  *out = NULL;
  if (n < 1 || p < 1 || ldx < n || prm->ntree < 1 || prm->nodesize < 1) return BFO_EINVAL;
  int32_t mtry = prm->mtry ? prm->mtry : (p / 3 > 1 ? p / 3 : 1);
  if (mtry < 1 || mtry > p) return BFO_EINVAL;
  if (prm->tree_begin < 0 || prm->tree_end > prm->ntree || prm->tree_begin > prm->tree_end) return BFO_EINVAL;
  int64_t ss = prm->sampsize ? prm->sampsize : n;
  if (ss < 1 || n >= ((int64_t)1 << 31) || ss >= ((int64_t)1 << 31)) return BFO_ERANGE;
  if (!prm->replace && ss != n) return BFO_ENOTIMPL;

  /* reading R17/R18: reject NaN/Inf, canonicalise -0.0 */
  double* Xc = (double*)malloc(sizeof(double) * (size_t)n * (size_t)p);
  if (!Xc) return BFO_ENOMEM;
  for (int32_t j = 0; j < p; j++)
    for (int64_t i = 0; i < n; i++) {
      double v = X[(int64_t)j * ldx + i];
      if (!isfinite(v)) { free(Xc); return BFO_ENONFINITE; }
      Xc[(int64_t)j * n + i] = canon(v);
    }
  int64_t* yq = (int64_t*)malloc(sizeof(int64_t) * (size_t)n);
  int32_t q = 0;
  int rc = bfo_fixed_point(y, n, ss, yq, &q);
  if (rc) { free(Xc); free(yq); return rc; }

  bfo_forest* F = (bfo_forest*)calloc(1, sizeof(bfo_forest));
  F->n = n; F->p = p; F->ntree = prm->ntree; F->tree_begin = prm->tree_begin; F->tree_end = prm->tree_end;
  F->q = q; F->mtry = mtry; F->nodesize = prm->nodesize; F->replace = prm->replace; F->sampsize = ss;
  F->seed = prm->seed;
  int nt = F->tree_end - F->tree_begin;
  F->trees = (otree*)calloc((size_t)(nt > 0 ? nt : 1), sizeof(otree));

  fit_job J;
  J.F = F; J.Xc = Xc; J.y = y; J.yq = yq; J.next = 0; J.err = 0;
  pthread_mutex_init(&J.mu, NULL);
  int nth = prm->nthreads > 0 ? prm->nthreads : 1;
  if (nth > nt) nth = nt > 0 ? nt : 1;
  pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * (size_t)nth);
  for (int k = 0; k < nth; k++) pthread_create(&th[k], NULL, fit_worker, &J);
  for (int k = 0; k < nth; k++) pthread_join(th[k], NULL);
  free(th);
  pthread_mutex_destroy(&J.mu);
  free(Xc);
  free(yq);
  if (J.err) { bfo_forest_free(F); return J.err; }
  *out = F;
  return BFO_OK;
}

void bfo_forest_free(bfo_forest* f) {
  if (!f) return;
  for (int i = 0; i < f->tree_end - f->tree_begin; i++) free(f->trees[i].nodes);
  free(f->trees);
  free(f);
}

int32_t bfo_forest_ntrees(const bfo_forest* f) { return f->tree_end - f->tree_begin; }
int32_t bfo_forest_q(const bfo_forest* f) { return f->q; }
int64_t bfo_tree_nnodes(const bfo_forest* f, int32_t i) { return f->trees[i].nnodes; }

int bfo_tree_export(const bfo_forest* f, int32_t i, int32_t* feature, double* thr, int32_t* left,
                    int64_t* count, double* value, double* drss) {
  if (i < 0 || i >= f->tree_end - f->tree_begin) return BFO_EINVAL;
  const otree* tr = &f->trees[i];
  for (int64_t k = 0; k < tr->nnodes; k++) {
    const onode* nd = &tr->nodes[k];
    if (feature) feature[k] = nd->feature;
    if (thr) thr[k] = nd->thr;
    if (left) left[k] = nd->left;
    if (count) count[k] = nd->count;
    if (value) value[k] = nd->value;
    if (drss) drss[k] = nd->drss;
  }
  return BFO_OK;
}

/* ------------------------------------------------------------------------ */
/* S5  Prediction: walk x_f <= thr -> left (eq.(2)); average trees.    */
/* ------------------------------------------------------------------------ */
static double tree_walk(const otree* tr, const double* x, int64_t ld, int64_t r) {
  int64_t k = 0;
  while (tr->nodes[k].feature >= 0) {
    const onode* nd = &tr->nodes[k];
    k = (x[(int64_t)nd->feature * ld + r] <= nd->thr) ? nd->left : nd->left + 1;
  }
  return tr->nodes[k].value;
}

int bfo_predict(const bfo_forest* f, const double* Xq, int64_t ldq, int64_t m, double* yhat_sum) {
  if (ldq < m) return BFO_EINVAL;
  for (int64_t r = 0; r < m; r++) {
    double s = 0.0;
    for (int i = 0; i < f->tree_end - f->tree_begin; i++) s += tree_walk(&f->trees[i], Xq, ldq, r);
    yhat_sum[r] = s;
  }
  return BFO_OK;
}

/* ------------------------------------------------------------------------ */
/* S7  Feistel permutation pi_tm on [0, n_o): 6 rounds, cycle walking.        */
/*     F_r(v) = x0 of Philox ctr (v, r, 3 | (m<<8), t).                       */
/* ------------------------------------------------------------------------ */
int64_t bfo_perm(uint64_t seed, int32_t t, int32_t m, int64_t n_o, int64_t a) {
  int b = 0;
  while (((int64_t)1 << b) < n_o) b++; /* ceil(log2 n_o) */
  if (b < 2) b = 2;
  if (b & 1) b++;
  int h = b / 2;
  uint32_t mask = (uint32_t)(((uint64_t)1 << h) - 1);
  uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
  uint64_t v = (uint64_t)a;
  do {
    uint32_t L = (uint32_t)(v >> h), R = (uint32_t)(v & mask);
    for (uint32_t r = 0; r < 6; r++) {
      uint32_t ctr[4] = {R, r, 3u | ((uint32_t)m << 8), (uint32_t)t};
      uint32_t x[4];
      bfo_philox4x32_10(ctr, key, x);
      uint32_t nR = L ^ (x[0] & mask);
      L = R;
      R = nR;
    }
    v = ((uint64_t)L << h) | R;
  } while ((int64_t)v >= n_o);
  return (int64_t)v;
}

/* ------------------------------------------------------------------------ */
/* S6-S8  OOB error, permutation importance, node purity.    */
/* ------------------------------------------------------------------------ */
int bfo_oob_importance(const bfo_forest* f, const double* X, int64_t ldx, const double* y,
                       int64_t n, int32_t p, int32_t perm_identity,
                       double* d_slots, double* npur_slots, double* oob_sum, int32_t* oob_cnt,
                       double* e_t, int64_t* nout_t) {
  if (n != f->n || p != f->p || ldx < n) return BFO_EINVAL;
  int nt = f->tree_end - f->tree_begin;
  int32_t* w = (int32_t*)malloc(sizeof(int32_t) * (size_t)n);
  int64_t* O = (int64_t*)malloc(sizeof(int64_t) * (size_t)n);
  double* xt = (double*)malloc(sizeof(double) * (size_t)p);
  char* used = (char*)malloc((size_t)p);
  for (int64_t i = 0; i < n; i++) { oob_sum[i] = 0.0; oob_cnt[i] = 0; }
  for (int i = 0; i < nt; i++) {
    int32_t t = f->tree_begin + i;
    const otree* tr = &f->trees[i];
    bfo_bootstrap(f->seed, t, n, f->sampsize, f->replace, w);
    int64_t no = 0;
    for (int64_t r = 0; r < n; r++)
      if (w[r] == 0) O[no++] = r; /* O_t ascending */
    nout_t[i] = no;
    /* e_t and OOB sums */
    double et = 0.0;
    for (int64_t a = 0; a < no; a++) {
      int64_t r = O[a];
      double fx = tree_walk(tr, X, ldx, r);
      oob_sum[r] += fx;
      oob_cnt[r] += 1;
      double d = y[r] - fx;
      et += d * d;
    }
    e_t[i] = et;
    /* features used by a split of t; IncNodePurity slots */
    for (int32_t m = 0; m < p; m++) { used[m] = 0; npur_slots[(int64_t)i * p + m] = 0.0; }
    for (int64_t k = 0; k < tr->nnodes; k++)
      if (tr->nodes[k].feature >= 0) {
        used[tr->nodes[k].feature] = 1;
        npur_slots[(int64_t)i * p + tr->nodes[k].feature] += tr->nodes[k].drss;
      }
    for (int32_t m = 0; m < p; m++) {
      double* dslot = &d_slots[(int64_t)i * p + m];
      if (!used[m] || no == 0) { *dslot = 0.0; continue; }
      double etm = 0.0;
      for (int64_t a = 0; a < no; a++) {
        int64_t r = O[a];
        int64_t pa = perm_identity ? a : bfo_perm(f->seed, t, m, no, a);
        for (int32_t j = 0; j < p; j++) xt[j] = X[(int64_t)j * ldx + r];
        xt[m] = X[(int64_t)m * ldx + O[pa]];
        double fx = tree_walk(tr, xt, 1, 0);
        double d = y[r] - fx;
        etm += d * d;
      }
      *dslot = (etm - et) / (double)no;
    }
  }
  free(w); free(O); free(xt); free(used);
  return BFO_OK;
}

int bfo_importance_finalize(const double* d_slots, const double* npur_slots, const double* oob_sum,
                            const int32_t* oob_cnt, const double* y, int64_t n, int32_t p, int32_t ntree,
                            double* inc_mse, double* inc_mse_raw, double* inc_mse_sd,
                            double* inc_node_purity, double* oob_mse, double* rsq) {
  if (ntree < 1 || n < 1 || p < 1) return BFO_EINVAL;
  for (int32_t m = 0; m < p; m++) {
    double raw = 0.0;
    for (int32_t t = 0; t < ntree; t++) raw += d_slots[(int64_t)t * p + m];
    raw /= (double)ntree;
    double v = 0.0;
    for (int32_t t = 0; t < ntree; t++) {
      double d = d_slots[(int64_t)t * p + m] - raw;
      v += d * d;
    }
    v /= (double)ntree;
    double sd = sqrt(v / (double)ntree);
    inc_mse_raw[m] = raw;
    inc_mse_sd[m] = sd;
    inc_mse[m] = (sd >= DBL_EPSILON) ? raw / sd : raw;
    double np = 0.0;
    for (int32_t t = 0; t < ntree; t++) np += npur_slots[(int64_t)t * p + m];
    inc_node_purity[m] = np / (double)ntree;
  }
  /* OOB MSE over rows with at least one OOB tree; rsq = 1 - mse/var_pop(y) */
  double se = 0.0;
  int64_t cnt = 0;
  for (int64_t i = 0; i < n; i++)
    if (oob_cnt[i] > 0) {
      double d = y[i] - oob_sum[i] / (double)oob_cnt[i];
      se += d * d;
      cnt++;
    }
  double mse = cnt ? se / (double)cnt : 0.0;
  double mean = 0.0;
  for (int64_t i = 0; i < n; i++) mean += y[i];
  mean /= (double)n;
  double var = 0.0;
  for (int64_t i = 0; i < n; i++) var += (y[i] - mean) * (y[i] - mean);
  var /= (double)n;
  *oob_mse = mse;
  *rsq = (var > 0.0) ? 1.0 - mse / var : 0.0;
  return BFO_OK;
}
