/*
 * oracle/cart_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, single-threaded CPU implementation of the Decision-Tree (CART)
 * regression hot path of Metz, Goli & Drechsler (IPDPS'23, dblp conf/ipps/MetzGD23):
 * fit, predict, MAPE / R^2 / adjusted-R^2 evaluation and leave-one-out refits.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this file's shared library.  The product path (the CUDA library under
 * paper_conf_ipps_metzgd23_b200/) shares no code, header, table or helper with it.
 *
 * Citations: "P:L" = /root/reference/PAPER.md line L (section / table / equation).
 * The paper names the model only ("Decision Tree regression", P:7),
 * gives the dataset row d = (y, p, c_1..c_m, t) (Eq. 1) and the accuracy
 * metrics MAPE, R^2 and adj. R^2 (Table II).  Everything else is a
 * reading recorded in DESIGN.md section "Readings" (R1..R18, numbered as SURVEY.md 8(c)
 * C1..C18 where they coincide).
 *
 * Arithmetic: IEEE fp64 round-to-nearest, compiled with -O2 -ffp-contract=off (no FMA
 * contraction) and no fast-math.  Sums are sequential Neumaier-compensated sums in the
 * fixed orders stated below.
 *
 * Pins (tests/test_oracle_*.py, all "-m 'not gpu'"):
 *   - split choice == exact-rational argmax of SSE_P - SSE_L - SSE_R (brute force)
 *   - depth-1 tree == optimum stump; depth<=3 greedy SSE >= optimum depth<=3 tree SSE
 *   - greedy tree == exact-arithmetic greedy recursion (tiny integer inputs)
 *   - invariants: leaf value = mean, SSE_L+SSE_R <= SSE_P, row multiset preserved,
 *     min_samples_leaf, depth bound, BFS links, training rows route to their leaf
 *   - metamorphic: y*2^k, row permutation (integer mode), truncation, duplicate column
 *   - scikit-learn DecisionTreeRegressor on tie-free continuous data (library routine)
 *   - metric closed forms (R^2 = 1 - SSE/SST, adj-R^2, yhat=y, yhat=mean)
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <float.h>

/* Output node: 48 bytes, BFS order, node 0 = root.  Declared here independently of the
 * product header include/dt.h (no shared headers); tests check the two layouts agree. */
typedef struct {
  int32_t feature;   /* split feature, -1 for a leaf */
  int32_t left;      /* left child index, -1 for a leaf */
  int32_t right;     /* right child index (= left + 1), -1 for a leaf */
  int32_t depth;     /* root = 0 */
  double threshold;  /* go left iff (double)x[feature] <= threshold; 0 for leaves */
  double value;      /* mean of y over the node's training rows */
  double impurity;   /* SSE / n_samples */
  int64_t n_samples;
} oracle_node;

/* ---------------------------------------------------------------- sums ---- */

/* Neumaier-compensated running sum (Reading R10: compensated fp64 in a fixed order). */
typedef struct { double s, c; } nsum;
static void ns_add(nsum* a, double v) {
  double t = a->s + v;
  if (fabs(a->s) >= fabs(v)) a->c += (a->s - t) + v;
  else a->c += (v - t) + a->s;
  a->s = t;
}
static double ns_val(const nsum* a) { return a->s + a->c; }

/* ---------------------------------------------------------------- fit ------ */

typedef struct {
  int64_t* rows;   /* row ids of the node, ascending */
  int64_t n;
  int32_t depth;
  int32_t id;      /* BFS index in the output */
} work_node;

static const float* g_X;  /* comparator context for qsort (single-threaded oracle) */
static int32_t g_d, g_f;
static int cmp_feature_then_row(const void* a, const void* b) {
  int64_t ra = *(const int64_t*)a, rb = *(const int64_t*)b;
  float xa = g_X[ra * g_d + g_f], xb = g_X[rb * g_d + g_f];
  if (xa < xb) return -1;           /* exact f32 compare: -0.0 == +0.0 (Reading R6) */
  if (xa > xb) return 1;
  return (ra < rb) ? -1 : (ra > rb);  /* ties by row id: canonical order (Reading R10) */
}

static int64_t floor_div_i64(int64_t a, int64_t b) {  /* b > 0 */
  int64_t q = a / b, r = a % b;
  return (r != 0 && r < 0) ? q - 1 : q;
}

/* Returns 0 on success, 1 on bad args, 2 on non-finite input, 3 on out of memory. */
int oracle_fit(const float* X, const double* y, int64_t n, int32_t d, int32_t max_depth,
               int64_t min_leaf, oracle_node** out_nodes, int64_t* out_count,
               int32_t* out_integer_mode, int64_t* out_split_evals) {
  if (n < 1 || d < 1 || d > 255 || max_depth < -1 || min_leaf < 1) return 1;
  for (int64_t i = 0; i < n * (int64_t)d; ++i) if (!isfinite(X[i])) return 2;
  double ymax_abs = 0.0;
  int integral = 1;
  for (int64_t i = 0; i < n; ++i) {
    if (!isfinite(y[i])) return 2;
    if (fabs(y[i]) > ymax_abs) ymax_abs = fabs(y[i]);
    if (floor(y[i]) != y[i]) integral = 0;
  }
  /* Reading R17 (integer mode): every y integral and max|y| * n < 2^52, so every
   * centered sum below is an exact integer < 2^53 in any order. */
  const int int_mode = integral && (ymax_abs * (double)n < 4503599627370496.0);
  if (out_integer_mode) *out_integer_mode = int_mode;

  int64_t cap_nodes = 2 * n + 1;  /* a binary tree with <= n leaves */
  oracle_node* nodes = (oracle_node*)calloc((size_t)cap_nodes, sizeof(oracle_node));
  work_node* queue = (work_node*)calloc((size_t)cap_nodes, sizeof(work_node));
  int64_t* sorted = (int64_t*)malloc(sizeof(int64_t) * (size_t)n);
  double* pre = (double*)malloc(sizeof(double) * (size_t)(n + 1));
  double* suf = (double*)malloc(sizeof(double) * (size_t)(n + 1));
  if (!nodes || !queue || !sorted || !pre || !suf) {
    free(nodes); free(queue); free(sorted); free(pre); free(suf);
    return 3;
  }
  g_X = X; g_d = d;

  int64_t head = 0, tail = 0, count = 1, split_evals = 0;
  queue[tail].rows = (int64_t*)malloc(sizeof(int64_t) * (size_t)n);
  for (int64_t i = 0; i < n; ++i) queue[tail].rows[i] = i;
  queue[tail].n = n; queue[tail].depth = 0; queue[tail].id = 0; ++tail;

  /* BFS: process nodes in queue order; a split appends left then right (Reading R9). */
  while (head < tail) {
    work_node w = queue[head++];
    const int64_t N = w.n;
    oracle_node* nd = &nodes[w.id];
    nd->depth = w.depth; nd->n_samples = N; nd->feature = -1; nd->left = -1; nd->right = -1;
    nd->threshold = 0.0;

    /* Node value = mean of its targets; sum in ascending row id (Reading R10). */
    nsum s = {0, 0};
    double ymin = y[w.rows[0]], ymax = y[w.rows[0]];
    for (int64_t k = 0; k < N; ++k) {
      double v = y[w.rows[k]];
      ns_add(&s, v);
      if (v < ymin) ymin = v;
      if (v > ymax) ymax = v;
    }
    const double sum = ns_val(&s);
    const double value = sum / (double)N;
    nsum q = {0, 0};
    for (int64_t k = 0; k < N; ++k) { double e = y[w.rows[k]] - value; ns_add(&q, e * e); }
    nd->value = value;
    nd->impurity = ns_val(&q) / (double)N;

    /* Leaf rules, in this order (Reading R8): depth limit, too few rows, pure node. */
    int leaf = 0;
    if (max_depth >= 0 && w.depth >= max_depth) leaf = 1;
    else if (N < 2 * min_leaf) leaf = 1;
    else if (ymin == ymax) leaf = 1;

    int32_t best_f = -1;
    int64_t best_i = -1;
    double best_gain = -1.0, best_t = 0.0;
    if (!leaf) {
      /* Center (Reading R10): integer mode c = floor(sum / N) exactly in int64,
       * real mode c = value.  All candidate sums are sums of (y - c). */
      double c = int_mode ? (double)floor_div_i64((int64_t)sum, N) : value;
      split_evals += N * (int64_t)d;  /* headline numerator: N*d per searched node */
      for (int32_t f = 0; f < d; ++f) {
        /* Order the node's rows by (x_f, row id). */
        memcpy(sorted, w.rows, sizeof(int64_t) * (size_t)N);
        g_f = f;
        qsort(sorted, (size_t)N, sizeof(int64_t), cmp_feature_then_row);
        /* S'_L(i): Neumaier prefix of (y - c) over the first i rows, forward.
         * S'_R(i): Neumaier suffix of (y - c) over rows i..N-1, backward. */
        nsum a = {0, 0};
        pre[0] = 0.0;
        for (int64_t k = 0; k < N; ++k) { ns_add(&a, y[sorted[k]] - c); pre[k + 1] = ns_val(&a); }
        nsum b = {0, 0};
        suf[N] = 0.0;
        for (int64_t k = N - 1; k >= 0; --k) { ns_add(&b, y[sorted[k]] - c); suf[k] = ns_val(&b); }
        for (int64_t i = 1; i < N; ++i) {
          float xlo = X[sorted[i - 1] * d + f], xhi = X[sorted[i] * d + f];
          /* Candidate i puts the first i rows left.  Valid iff the f32 values differ
           * and both children keep >= min_samples_leaf rows (Reading R6, R2). */
          if (!(xlo < xhi) || i < min_leaf || N - i < min_leaf) continue;
          /* Gain = SSE_P - SSE_L - SSE_R = (n_L n_R / N)(m_L - m_R)^2
           *      = (S'_L n_R - S'_R n_L)^2 / (N n_L n_R)          (Reading R19). */
          double nl = (double)i, nr = (double)(N - i), Nd = (double)N;
          double D = pre[i] * nr - suf[i] * nl;
          double gain = (D * D) / ((Nd * nl) * nr);
          /* Strictly greater: lowest feature, then lowest threshold on ties (R4). */
          if (gain > best_gain) {
            best_gain = gain; best_f = f; best_i = i;
            /* Midpoint threshold in fp64 (Reading R5). */
            best_t = (double)xlo / 2.0 + (double)xhi / 2.0;
          }
        }
      }
      if (best_f < 0) leaf = 1;  /* no valid candidate */
    }
    if (leaf) { free(w.rows); continue; }

    /* Split even if best_gain == 0 (node not pure; Reading R8). */
    nd->feature = best_f; nd->threshold = best_t;
    nd->left = (int32_t)count; nd->right = (int32_t)(count + 1);
    int64_t nL = best_i, nR = N - best_i;
    int64_t* lrows = (int64_t*)malloc(sizeof(int64_t) * (size_t)nL);
    int64_t* rrows = (int64_t*)malloc(sizeof(int64_t) * (size_t)nR);
    /* Children keep ascending row-id order: filter the parent's row list by x <= t. */
    int64_t li = 0, ri = 0;
    for (int64_t k = 0; k < N; ++k) {
      int64_t r = w.rows[k];
      if ((double)X[r * d + best_f] <= best_t) lrows[li++] = r; else rrows[ri++] = r;
    }
    free(w.rows);
    if (li != nL || ri != nR) {  /* cannot happen: x_lo <= t < x_hi (Reading R5) */
      free(lrows); free(rrows);
      for (int64_t k = head; k < tail; ++k) free(queue[k].rows);
      free(nodes); free(queue); free(sorted); free(pre); free(suf);
      return 4;
    }
    queue[tail].rows = lrows; queue[tail].n = nL; queue[tail].depth = w.depth + 1;
    queue[tail].id = (int32_t)count; ++tail;
    queue[tail].rows = rrows; queue[tail].n = nR; queue[tail].depth = w.depth + 1;
    queue[tail].id = (int32_t)(count + 1); ++tail;
    count += 2;
  }
  free(queue); free(sorted); free(pre); free(suf);
  *out_nodes = nodes;
  *out_count = count;
  if (out_split_evals) *out_split_evals = split_evals;
  return 0;
}

void oracle_free(void* p) { free(p); }

/* ---------------------------------------------------------------- predict -- */

/* From the root, go left iff (double)x[f] <= threshold, until a leaf (Reading R5). */
void oracle_predict(const oracle_node* nodes, int64_t count, const float* X, int64_t n,
                    int32_t d, double* yhat) {
  (void)count;
  for (int64_t r = 0; r < n; ++r) {
    int32_t k = 0;
    while (nodes[k].feature >= 0) {
      double x = (double)X[r * d + nodes[k].feature];
      k = (x <= nodes[k].threshold) ? nodes[k].left : nodes[k].right;
    }
    yhat[r] = nodes[k].value;
  }
}

/* ---------------------------------------------------------------- eval ----- */

/* MAPE, R^2, adjusted R^2 (Table II; Readings R12-R14).
 * out[0] = MAPE as a fraction, out[1] = R^2, out[2] = adj-R^2 (NaN if n-p-1 <= 0). */
void oracle_eval(const double* y, const double* yhat, int64_t n, int32_t p, double* out) {
  nsum ape = {0, 0}, sse = {0, 0}, sy = {0, 0}, sst = {0, 0};
  for (int64_t i = 0; i < n; ++i) {
    double den = fabs(y[i]);
    if (den < DBL_EPSILON) den = DBL_EPSILON;
    ns_add(&ape, fabs(y[i] - yhat[i]) / den);
    double e = y[i] - yhat[i];
    ns_add(&sse, e * e);
    ns_add(&sy, y[i]);
  }
  double ybar = ns_val(&sy) / (double)n;
  for (int64_t i = 0; i < n; ++i) { double e = y[i] - ybar; ns_add(&sst, e * e); }
  double SSE = ns_val(&sse), SST = ns_val(&sst);
  double r2;
  if (SST == 0.0) r2 = (SSE == 0.0) ? 1.0 : 0.0;  /* sklearn force_finite rule (R13) */
  else r2 = 1.0 - SSE / SST;
  double adj;
  if ((double)n - (double)p - 1.0 <= 0.0) adj = NAN;
  else adj = 1.0 - (1.0 - r2) * ((double)n - 1.0) / ((double)n - (double)p - 1.0);
  out[0] = ns_val(&ape) / (double)n;
  out[1] = r2;
  out[2] = adj;
}

/* ---------------------------------------------------------------- LOO ------ */

/* Leave-one-out (Reading R11): for each i, fit on the other n-1 rows in their original
 * relative order, predict row i.  Returns the out-of-fold predictions in yhat_oof. */
int oracle_loo(const float* X, const double* y, int64_t n, int32_t d, int32_t max_depth,
               int64_t min_leaf, double* yhat_oof) {
  if (n < 2) return 1;
  float* Xs = (float*)malloc(sizeof(float) * (size_t)((n - 1) * d));
  double* ys = (double*)malloc(sizeof(double) * (size_t)(n - 1));
  if (!Xs || !ys) { free(Xs); free(ys); return 3; }
  for (int64_t i = 0; i < n; ++i) {
    int64_t k = 0;
    for (int64_t r = 0; r < n; ++r) {
      if (r == i) continue;
      memcpy(Xs + k * d, X + r * d, sizeof(float) * (size_t)d);
      ys[k] = y[r];
      ++k;
    }
    oracle_node* nodes = NULL; int64_t cnt = 0; int32_t im = 0;
    int st = oracle_fit(Xs, ys, n - 1, d, max_depth, min_leaf, &nodes, &cnt, &im, NULL);
    if (st) { free(Xs); free(ys); return st; }
    oracle_predict(nodes, cnt, X + i * d, 1, d, &yhat_oof[i]);
    free(nodes);
  }
  free(Xs); free(ys);
  return 0;
}

/* ---------------------------------------------------------------- importances */

/* NEXT-1 (Table III; Reading R3): mean decrease in SSE per feature,
 * normalised to sum 1: imp[f] = sum over internal nodes with feature f of
 * N*imp_P - N_L*imp_L - N_R*imp_R. */
void oracle_importances(const oracle_node* nodes, int64_t count, int32_t d, double* imp) {
  for (int32_t f = 0; f < d; ++f) imp[f] = 0.0;
  for (int64_t k = 0; k < count; ++k) {
    const oracle_node* a = &nodes[k];
    if (a->feature < 0) continue;
    const oracle_node* l = &nodes[a->left];
    const oracle_node* r = &nodes[a->right];
    imp[a->feature] += (double)a->n_samples * a->impurity - (double)l->n_samples * l->impurity -
                       (double)r->n_samples * r->impurity;
  }
  double tot = 0.0;
  for (int32_t f = 0; f < d; ++f) tot += imp[f];
  if (tot > 0.0) for (int32_t f = 0; f < d; ++f) imp[f] /= tot;
}

/* ------------------------------------------------------- random forest (NEXT-2) -- */

/* Random Forest = bagged CART ("the Random Forest Tree is an ensemble of Decision
 * Trees"; "the decision is taken based on the average value of all included
 * Decision Trees").  Reading R20: tree t is grown by oracle_fit on the bootstrap sample
 * X[idx_t], y[idx_t] (n draws with replacement, in draw order; duplicates count towards
 * min_samples_leaf); every split considers all d features (sklearn's regression default,
 * max_features = 1.0).  Draw i of tree t (counter-based SplitMix64, Reading R21):
 *   z = seed + 0x9E3779B97F4A7C15 * ((t << 32) + i + 1)   (mod 2^64)
 *   z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9; z = (z ^ (z >> 27)) * 0x94D049BB133111EB;
 *   z ^= z >> 31;  idx = z mod n. */
void oracle_bootstrap(uint64_t seed, int32_t t, int64_t n, uint32_t* idx) {
  for (int64_t i = 0; i < n; ++i) {
    uint64_t z = seed + 0x9E3779B97F4A7C15ull * ((((uint64_t)(uint32_t)t) << 32) + (uint64_t)i + 1ull);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    z ^= z >> 31;
    idx[i] = (uint32_t)(z % (uint64_t)n);
  }
}

/* Forest prediction: the mean of the trees' predictions, summed in tree order (plain
 * fp64, no compensation: T is small), then divided by T. */
void oracle_forest_predict(const oracle_node* const* trees, const int64_t* counts, int32_t n_trees,
                           const float* X, int64_t n, int32_t d, double* yhat) {
  for (int64_t r = 0; r < n; ++r) {
    double acc = 0.0;
    for (int32_t t = 0; t < n_trees; ++t) {
      double v;
      oracle_predict(trees[t], counts[t], X + r * d, 1, d, &v);
      acc = acc + v;
    }
    yhat[r] = acc / (double)n_trees;
  }
}

/* ------------------------------------------------------- K-nearest neighbours (NEXT-4) */

/* KNN regression ("K-Nearest Neighbors ... non-linear dependencies", Table II
 * P:214; sklearn KNeighborsRegressor defaults: k = 5, uniform weights, Euclidean).
 * Reading R22: dist(q, x) = sum over f = 0..d-1, in feature order, of (q_f - x_f)^2,
 * each term fused into the running sum: acc = fma(q_f - x_f, q_f - x_f, acc), with
 * q_f - x_f taken in fp64 from the f32 inputs (one rounding).  Squared distance orders
 * exactly like the Euclidean one.  Neighbours: the k training rows with the smallest
 * (dist, row index) -- ties go to the lower index; yhat = (sum of their y in that
 * order) / k.  k <= n_train. */
void oracle_knn(const float* Xtr, const double* ytr, int64_t ntr, int32_t d, const float* Xq,
                int64_t nq, int32_t k, double* yhat) {
  double* bd = (double*)malloc(sizeof(double) * (size_t)k);
  int64_t* bi = (int64_t*)malloc(sizeof(int64_t) * (size_t)k);
  for (int64_t q = 0; q < nq; ++q) {
    int32_t cnt = 0;  /* bd/bi sorted ascending by (dist, index) */
    for (int64_t r = 0; r < ntr; ++r) {
      double acc = 0.0;
      for (int32_t f = 0; f < d; ++f) {
        double df = (double)Xq[q * d + f] - (double)Xtr[r * d + f];
        acc = fma(df, df, acc);
      }
      if (cnt == k && !(acc < bd[k - 1])) continue;  /* equal distance: the lower index stays */
      int32_t pos = (cnt < k) ? cnt : k - 1;
      while (pos > 0 && acc < bd[pos - 1]) {  /* strict: earlier (lower) index first on ties */
        bd[pos] = bd[pos - 1];
        bi[pos] = bi[pos - 1];
        --pos;
      }
      bd[pos] = acc;
      bi[pos] = r;
      if (cnt < k) ++cnt;
    }
    double s = 0.0;
    for (int32_t j = 0; j < k; ++j) s = s + ytr[bi[j]];
    yhat[q] = s / (double)k;
  }
  free(bd);
  free(bi);
}
