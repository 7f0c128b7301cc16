// Leave-one-out refits for the paper-sized table (BASELINE configs[0]: 40 (CNN, GPU) rows
// x 4 features; the paper's 70/30 split, has no seed -> Reading R11).
// One CTA per fold: the fold's n-1 rows, their per-feature orders and the whole tree
// live in shared memory; level-synchronous BFS; the held-out row is predicted at the end.  The split rule is
// the one of dt_fit (Readings R1-R10, R19).  Within a node the per-feature prefix and
// suffix sums run sequentially in (x, row id) order with Neumaier compensation.
#include <math.h>

#include "dt_internal.cuh"

namespace dtl {

namespace {

constexpr int kMaxN = 64;
constexpr int kMaxD = 32;
constexpr int kMaxNodes = 2 * kMaxN;

struct TNode {
  int32_t feature, left;
  int32_t depth, n;
  double thr, value;
};

__device__ __forceinline__ void nadd(double& s, double& c, double v) {
  const double t = __dadd_rn(s, v);
  if (fabs(s) >= fabs(v)) c = __dadd_rn(c, __dadd_rn(__dsub_rn(s, t), v));
  else c = __dadd_rn(c, __dadd_rn(__dsub_rn(v, t), s));
  s = t;
}

__device__ __forceinline__ long long fdiv(long long a, long long b) {
  long long q = a / b, r = a % b;
  return (r != 0 && r < 0) ? q - 1 : q;
}

__global__ void __launch_bounds__(256)
loo_kernel(const float* __restrict__ Xg, const double* __restrict__ yg, int n_all, int d,
           int max_depth, long long min_leaf, double* __restrict__ yhat) {
  __shared__ float X[kMaxN * kMaxD];
  __shared__ double y[kMaxN];
  __shared__ uint8_t order[kMaxD][kMaxN];  // rows of feature f in (x, row) order
  __shared__ int16_t nid[kMaxN];           // current node of each row
  __shared__ TNode tree[kMaxNodes];
  // per (splittable node of the level, feature): best gain, position, threshold
  __shared__ double bgain[kMaxN / 2 * kMaxD];
  __shared__ int bpos[kMaxN / 2 * kMaxD];
  __shared__ double bthr[kMaxN / 2 * kMaxD];
  __shared__ uint8_t s_leafv[kMaxN], s_split[kMaxN];
  __shared__ double s_cc[kMaxN];
  __shared__ int s_int_mode, s_count, s_nsplit;

  const int fold = blockIdx.x;
  const int n = n_all - 1;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  // fold's training rows, original relative order
  for (int i = tid; i < n * d; i += blockDim.x) {
    const int r = i / d, f = i - r * d;
    const int src = r < fold ? r : r + 1;
    X[i] = Xg[src * d + f];
  }
  for (int r = tid; r < n; r += blockDim.x) {
    y[r] = yg[r < fold ? r : r + 1];
    nid[r] = 0;
  }
  __syncthreads();
  // per-feature order by (x, row): rank sort
  for (int i = tid; i < n * d; i += blockDim.x) {
    const int f = i / n, r = i - f * n;
    const float xr = X[r * d + f];
    int rank = 0;
    for (int q = 0; q < n; ++q) {
      const float xq = X[q * d + f];
      rank += (xq < xr) || (xq == xr && q < r);
    }
    order[f][rank] = (uint8_t)r;
  }
  if (tid == 0) {
    double amax = 0.0;
    int integral = 1;
    for (int r = 0; r < n; ++r) {
      amax = fmax(amax, fabs(y[r]));
      if (floor(y[r]) != y[r]) integral = 0;
    }
    s_int_mode = integral && amax * (double)n < 4503599627370496.0;
    tree[0].depth = 0;
    tree[0].n = n;
    s_count = 1;
  }
  __syncthreads();

  // Level-synchronous BFS: the nodes of one depth [lo, hi) are evaluated together
  // (statistics: a thread per node; split scans: a thread per (node, feature); the
  // choice and the BFS numbering of the children: one thread, in node order; the
  // partition: a thread per row).  Per node and feature the arithmetic is the sequential
  // sequential reading R10 (Neumaier sums in (x, row) order), so the trees are identical.
  int lo = 0, hi = 1;
  while (lo < hi) {
    const int nn = hi - lo;
    for (int q = tid; q < nn; q += blockDim.x) {
      const int node = lo + q;
      double s = 0, c = 0, mn = INFINITY, mx = -INFINITY;
      int N = 0;
      for (int r = 0; r < n; ++r)
        if (nid[r] == node) { nadd(s, c, y[r]); mn = fmin(mn, y[r]); mx = fmax(mx, y[r]); ++N; }
      const double sum = __dadd_rn(s, c);
      const double value = __ddiv_rn(sum, (double)N);
      TNode& t = tree[node];
      t.n = N;
      t.value = value;
      t.feature = -1;
      t.left = -1;
      t.thr = 0.0;
      int leaf = 0;
      if (max_depth >= 0 && t.depth >= max_depth) leaf = 1;
      else if ((long long)N < 2 * min_leaf) leaf = 1;
      else if (mn == mx) leaf = 1;
      s_leafv[q] = (uint8_t)leaf;
      s_cc[q] = s_int_mode ? (double)fdiv((long long)sum, (long long)N) : value;
    }
    __syncthreads();
    if (tid == 0) {  // the level's splittable nodes, in node order
      int m = 0;
      for (int q = 0; q < nn; ++q)
        if (!s_leafv[q]) s_split[m++] = (uint8_t)q;
      s_nsplit = m;
    }
    __syncthreads();
    const int ns = s_nsplit;
    for (int pidx = tid; pidx < ns * d; pidx += blockDim.x) {
      const int q = s_split[pidx / d], f = pidx - (pidx / d) * d;
      const int node = lo + q;
      const double cc = s_cc[q];
      int rows[kMaxN];
      int m = 0;
      for (int k = 0; k < n; ++k) {
        const int r = order[f][k];
        if (nid[r] == node) rows[m++] = r;
      }
      double pre[kMaxN + 1], suf[kMaxN + 1];
      double s = 0, c = 0;
      pre[0] = 0.0;
      for (int k = 0; k < m; ++k) { nadd(s, c, __dsub_rn(y[rows[k]], cc)); pre[k + 1] = __dadd_rn(s, c); }
      s = 0; c = 0;
      suf[m] = 0.0;
      for (int k = m - 1; k >= 0; --k) { nadd(s, c, __dsub_rn(y[rows[k]], cc)); suf[k] = __dadd_rn(s, c); }
      double bg = -1.0, bt = 0.0;
      int bp = -1;
      for (int i = 1; i < m; ++i) {
        const float xlo = X[rows[i - 1] * d + f], xhi = X[rows[i] * d + f];
        if (!(xlo < xhi) || (long long)i < min_leaf || (long long)(m - i) < min_leaf) continue;
        const double nl = (double)i, nr = (double)(m - i), Nd = (double)m;
        const double D = __dsub_rn(__dmul_rn(pre[i], nr), __dmul_rn(suf[i], nl));
        const double g = __ddiv_rn(__dmul_rn(D, D), __dmul_rn(__dmul_rn(Nd, nl), nr));
        if (g > bg) {
          bg = g;
          bp = i;
          bt = __dadd_rn(__ddiv_rn((double)xlo, 2.0), __ddiv_rn((double)xhi, 2.0));
        }
      }
      bgain[pidx] = bg;
      bpos[pidx] = bp;
      bthr[pidx] = bt;
    }
    __syncthreads();
    if (tid == 0) {  // choices and children ids in node order (BFS numbering)
      for (int u = 0; u < ns; ++u) {
        int bf = -1;
        double bg = -1.0;
        for (int f = 0; f < d; ++f)
          if (bpos[u * d + f] >= 0 && bgain[u * d + f] > bg) { bg = bgain[u * d + f]; bf = f; }
        if (bf >= 0) {
          TNode& t = tree[lo + s_split[u]];
          t.feature = bf;
          t.thr = bthr[u * d + bf];
          t.left = s_count;
          tree[s_count].depth = t.depth + 1;
          tree[s_count + 1].depth = t.depth + 1;
          s_count += 2;
        }
      }
    }
    __syncthreads();
    for (int r = tid; r < n; r += blockDim.x) {  // the level's partition
      const int node = nid[r];
      if (node >= lo && node < hi && tree[node].feature >= 0) {
        const TNode& t = tree[node];
        nid[r] = (int16_t)(((double)X[r * d + t.feature] <= t.thr) ? t.left : t.left + 1);
      }
    }
    lo = hi;
    hi = s_count;
    __syncthreads();
  }
  // predict the held-out row
  if (tid == 0) {
    int k = 0;
    while (tree[k].feature >= 0) {
      const double x = (double)Xg[fold * d + tree[k].feature];
      k = (x <= tree[k].thr) ? tree[k].left : tree[k].left + 1;
    }
    yhat[fold] = tree[k].value;
  }
}

}  // namespace

dt_status loo_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t max_depth,
                   int64_t min_leaf, double* yhat, cudaStream_t s) {
  const int pr = prof_begin(PK_LOO, s, 1);
  loo_kernel<<<(unsigned)n, 256, 0, s>>>(X, y, (int)n, d, max_depth, (long long)min_leaf, yhat);
  prof_end(pr, s, (4.0 * d + 8.0) * (double)n + 8.0 * (double)n);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

}  // namespace dtl
