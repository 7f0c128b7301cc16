// Batched tree prediction (the PM's estimate over DSE candidate sets, PAPER.md:205,
// :245-247) and the fused accuracy metrics (MAPE, R^2, adj-R^2; Table II
// :211-217).  HBM-bound: 4d B read + 8 B written per prediction; 16 B per metric element.
#include <math.h>
#include <stdlib.h>

#include <algorithm>

#include "dt_internal.cuh"

namespace dtl {

namespace {

constexpr int kMaxSmemNodes = (227 * 1024) / 8;

// One traversal step: go left iff !(x > RD32(t)); for finite x this is exactly
// (double)x <= t (Reading R5).  Leaves self-loop (+inf threshold, left = self).
__device__ __forceinline__ uint32_t step(uint2 nd, const float* __restrict__ xr) {
  const uint32_t f = nd.y >> 24;
  const uint32_t left = nd.y & 0xFFFFFFu;
  const float x = __ldg(xr + f);
  return (x > __uint_as_float(nd.x)) ? left + 1 : left;
}

// kThr threads x kRPT rows in flight per CTA: every row's features are re-read at each of
// the `depth` levels, so the CTA's rows (kThr * kRPT * 4d bytes) must stay L1-resident
// next to the smem tree; the host picks (kThr, kRPT) and the smem carveout accordingly.
template <bool kSmem, int kThr, int kRowsPerThread>
__global__ void __launch_bounds__(kThr)
predict_kernel(const uint2* __restrict__ gnodes, const double* __restrict__ value, int count,
               int depth, const float* __restrict__ X, int64_t n, int d,
               double* __restrict__ yhat) {
  extern __shared__ uint2 snodes[];
  if (kSmem) {
    for (int i = threadIdx.x; i < count; i += blockDim.x) snodes[i] = gnodes[i];
    __syncthreads();
  }
  const uint2* nodes = kSmem ? snodes : gnodes;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x * kRowsPerThread;
  for (int64_t base = ((int64_t)blockIdx.x * blockDim.x) * kRowsPerThread + threadIdx.x;
       base < n; base += stride) {
    uint32_t k[kRowsPerThread];
    const float* xr[kRowsPerThread];
#pragma unroll
    for (int j = 0; j < kRowsPerThread; ++j) {
      int64_t r = base + (int64_t)j * blockDim.x;
      if (r >= n) r = n - 1;  // duplicate work on the tail, never stored
      xr[j] = X + r * d;
      k[j] = 0;
    }
    for (int l = 0; l < depth; ++l) {
#pragma unroll
      for (int j = 0; j < kRowsPerThread; ++j) k[j] = step(nodes[k[j]], xr[j]);
    }
#pragma unroll
    for (int j = 0; j < kRowsPerThread; ++j) {
      int64_t r = base + (int64_t)j * blockDim.x;
      if (r < n) yhat[r] = __ldg(value + k[j]);
    }
  }
}

// Column predict: thread t keeps its current row in shared-memory column t (feature-major
// s[f][t]), so both the 16/32 stores and the data-dependent feature reads of a warp are
// bank-conflict-free; the next row is prefetched into registers (four or eight 128-bit
// loads) during the traversal.  No block barrier after the tree load.
template <int kThr, int kD, int kR>
__global__ void __launch_bounds__(kThr)
predict_col_kernel(const uint2* __restrict__ gnodes, const double* __restrict__ value, int count,
                   int depth, const float* __restrict__ X, int64_t n, double* __restrict__ yhat) {
  extern __shared__ uint2 sm[];
  uint2* tree = sm;
  // kR columns per thread: column j of thread t at cols[(j * kD + f) * kThr + t]
  float* cols = reinterpret_cast<float*>(sm + count) + threadIdx.x;
  for (int i = threadIdx.x; i < count; i += kThr) tree[i] = gnodes[i];
  __syncthreads();
  const int64_t stride = (int64_t)gridDim.x * kThr * kR;
  float4 nx[kR][kD / 4];
  auto fetch = [&](int64_t base) {
#pragma unroll
    for (int j = 0; j < kR; ++j) {
      const int64_t rr = base + j * kThr;
      if (rr < n) {
        const float4* src = reinterpret_cast<const float4*>(X + rr * kD);
#pragma unroll
        for (int q = 0; q < kD / 4; ++q) nx[j][q] = __ldcs(src + q);
      }
    }
  };
  int64_t base = (int64_t)blockIdx.x * kThr * kR + threadIdx.x;
  if (base < n) fetch(base);
  for (; base < n; base += stride) {
#pragma unroll
    for (int j = 0; j < kR; ++j)
#pragma unroll
      for (int q = 0; q < kD / 4; ++q) {
        float* c = cols + (j * kD + 4 * q) * kThr;
        c[0] = nx[j][q].x;
        c[kThr] = nx[j][q].y;
        c[2 * kThr] = nx[j][q].z;
        c[3 * kThr] = nx[j][q].w;
      }
    if (base + stride < n) fetch(base + stride);
    uint32_t k[kR];
#pragma unroll
    for (int j = 0; j < kR; ++j) k[j] = 0;
    for (int l = 0; l < depth; ++l) {
#pragma unroll
      for (int j = 0; j < kR; ++j) {
        const uint2 nd = tree[k[j]];
        const uint32_t left = nd.y & 0xFFFFFFu;
        k[j] = (cols[(j * kD + (nd.y >> 24)) * kThr] > __uint_as_float(nd.x)) ? left + 1 : left;
      }
    }
#pragma unroll
    for (int j = 0; j < kR; ++j) {
      const int64_t rr = base + j * kThr;
      if (rr < n) yhat[rr] = __ldg(value + k[j]);
    }
  }
}

// ----------------------------------------------------------------------------- eval --

struct Part {  // per-block partial: sums + Welford/Chan moments of y
  double ape, sse, cnt, mean, m2;
};

__device__ __forceinline__ void chan_merge(double& na, double& ma, double& Ma, double nb,
                                           double mb, double Mb) {
  if (nb == 0.0) return;
  if (na == 0.0) {
    na = nb; ma = mb; Ma = Mb;
    return;
  }
  const double n = na + nb;
  const double delta = mb - ma;
  ma = ma + delta * (nb / n);
  Ma = Ma + Mb + delta * delta * (na * nb / n);
  na = n;
}

__device__ __forceinline__ void part_merge(Part& a, const Part& b) {
  a.ape += b.ape;
  a.sse += b.sse;
  chan_merge(a.cnt, a.mean, a.m2, b.cnt, b.mean, b.m2);
}

__device__ __forceinline__ Part shfl_part(const Part& p, int off) {
  Part q;
  q.ape = __shfl_down_sync(0xffffffffu, p.ape, off);
  q.sse = __shfl_down_sync(0xffffffffu, p.sse, off);
  q.cnt = __shfl_down_sync(0xffffffffu, p.cnt, off);
  q.mean = __shfl_down_sync(0xffffffffu, p.mean, off);
  q.m2 = __shfl_down_sync(0xffffffffu, p.m2, off);
  return q;
}

// Fixed-shape block reduction (deterministic for a fixed blockDim).
__device__ Part block_reduce(Part p) {
  __shared__ Part sh[32];
  for (int off = 16; off > 0; off >>= 1) {
    Part q = shfl_part(p, off);
    part_merge(p, q);
  }
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) sh[w] = p;
  __syncthreads();
  const int nw = (blockDim.x + 31) >> 5;
  if (w == 0) {
    p = (lane < nw) ? sh[lane] : Part{0, 0, 0, 0, 0};
    for (int off = 16; off > 0; off >>= 1) {
      Part q = shfl_part(p, off);
      part_merge(p, q);
    }
  }
  return p;
}

template <bool kFused>
__global__ void __launch_bounds__(256)
eval_partial_kernel(const double* __restrict__ y, const double* __restrict__ yhat,
                    const uint2* __restrict__ nodes, const double* __restrict__ value,
                    int depth, const float* __restrict__ X, int d, int64_t n, int64_t chunk,
                    Part* __restrict__ parts) {
  const int64_t lo = (int64_t)blockIdx.x * chunk;
  const int64_t hi = min(n, lo + chunk);
  Part p{0, 0, 0, 0, 0};
  for (int64_t r = lo + threadIdx.x; r < hi; r += blockDim.x) {
    const double yr = y[r];
    double yh;
    if (kFused) {
      const float* xr = X + r * d;
      uint32_t k = 0;
      for (int l = 0; l < depth; ++l) k = step(nodes[k], xr);
      yh = __ldg(value + k);
    } else {
      yh = yhat[r];
    }
    const double e = yr - yh;
    const double den = fmax(fabs(yr), 2.220446049250313e-16);  // max(|y|, DBL_EPSILON), R12
    p.ape += __ddiv_rn(fabs(e), den);
    p.sse += __dmul_rn(e, e);
    // Welford update of (n, mean, M2) of y
    p.cnt += 1.0;
    const double delta = yr - p.mean;
    p.mean += __ddiv_rn(delta, p.cnt);
    p.m2 += __dmul_rn(delta, yr - p.mean);
  }
  p = block_reduce(p);
  if (threadIdx.x == 0) parts[blockIdx.x] = p;
}

__global__ void __launch_bounds__(1024)
eval_final_kernel(const Part* __restrict__ parts, int nparts, int64_t n, int p_pred,
                  double* __restrict__ out) {
  Part acc{0, 0, 0, 0, 0};
  for (int i = threadIdx.x; i < nparts; i += blockDim.x) part_merge(acc, parts[i]);
  acc = block_reduce(acc);
  if (threadIdx.x == 0) {
    const double nn = (double)n;
    const double sst = acc.m2;
    double r2;
    if (sst == 0.0) r2 = (acc.sse == 0.0) ? 1.0 : 0.0;  // Reading R13
    else r2 = 1.0 - acc.sse / sst;
    double adj;
    if (nn - (double)p_pred - 1.0 <= 0.0) adj = __longlong_as_double(0x7ff8000000000000ll);
    else adj = 1.0 - (1.0 - r2) * (nn - 1.0) / (nn - (double)p_pred - 1.0);  // R14
    out[0] = acc.ape / nn;
    out[1] = r2;
    out[2] = adj;
  }
}

// Merges a rank's block partials into ONE partial (fixed shape), for the allgather of
// dt_eval_sharded.
__global__ void __launch_bounds__(1024) eval_local_kernel(const Part* __restrict__ parts, int nparts,
                                                          Part* __restrict__ out) {
  Part acc{0, 0, 0, 0, 0};
  for (int i = threadIdx.x; i < nparts; i += blockDim.x) part_merge(acc, parts[i]);
  acc = block_reduce(acc);
  if (threadIdx.x == 0) *out = acc;
}

// The ranks' partials merged in rank order (every rank runs the same sequence, so every
// rank gets bitwise the same metrics); n = the merged count.
__global__ void eval_ranks_kernel(const Part* __restrict__ parts, int world, int p_pred, double* __restrict__ out) {
  if (threadIdx.x != 0) return;
  Part acc{0, 0, 0, 0, 0};
  for (int r = 0; r < world; ++r) part_merge(acc, parts[r]);
  const double nn = acc.cnt;
  double r2;
  if (acc.m2 == 0.0) r2 = (acc.sse == 0.0) ? 1.0 : 0.0;  // Reading R13
  else r2 = 1.0 - acc.sse / acc.m2;
  double adj;
  if (nn - (double)p_pred - 1.0 <= 0.0) adj = __longlong_as_double(0x7ff8000000000000ll);
  else adj = 1.0 - (1.0 - r2) * (nn - 1.0) / (nn - (double)p_pred - 1.0);  // R14
  out[0] = acc.ape / nn;
  out[1] = r2;
  out[2] = adj;
  out[3] = nn;
}

template <bool kSmem, int kThr, int kRPT>
dt_status launch_predict(const dt_tree* t, const float* X, int64_t n, int32_t d, double* yhat,
                         cudaStream_t s, int carveout) {
  const size_t smem = kSmem ? sizeof(uint2) * (size_t)t->count : 0;
  auto kern = predict_kernel<kSmem, kThr, kRPT>;
  if (kSmem) DT_CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  DT_CK(cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, carveout));
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kThr, smem);
  if (per_sm < 1) per_sm = 1;
  const int64_t need = (n + (int64_t)kThr * kRPT - 1) / ((int64_t)kThr * kRPT);
  const int64_t g = std::min<int64_t>((int64_t)num_sms() * per_sm, std::max<int64_t>(1, need));
  kern<<<(unsigned)g, kThr, smem, s>>>(t->dev_packed, t->dev_value, (int)t->count, t->depth, X, n, d, yhat);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

// ------------------------------------------------------------ multi-depth eval (C5) --

// One pass over held-out rows evaluates EVERY truncation depth 0..D of a tree at once:
// the depth-l truncation predicts the value of the node the row reaches after l steps
// (or of the leaf it stopped at).  Per-depth MAPE / SSE partials plus Welford moments of
// y, fixed-shape reductions (deterministic).  Greedy CART fits are prefix-consistent,
// fit(D', m) == truncate(fit(D, m), D') (tests), so a (max_depth x m) grid
// needs one deep fit per m and this pass (BASELINE configs[4]).
constexpr int kMaxEvalDepth = 32;

struct DepthPart {
  double ape[kMaxEvalDepth + 1];
  double sse[kMaxEvalDepth + 1];
  double cnt, mean, m2;
};

__global__ void __launch_bounds__(256)
eval_depths_partial_kernel(const uint2* __restrict__ nodes, const double* __restrict__ value, int depth,
                           const float* __restrict__ X, int d, const double* __restrict__ y, int64_t n,
                           int64_t chunk, DepthPart* __restrict__ parts) {
  __shared__ double sh_ape[8][kMaxEvalDepth + 1];
  __shared__ double sh_sse[8][kMaxEvalDepth + 1];
  __shared__ Part sh_y[32];
  const int64_t lo = (int64_t)blockIdx.x * chunk, hi = min(n, lo + chunk);
  double ape[kMaxEvalDepth + 1], sse[kMaxEvalDepth + 1];
#pragma unroll
  for (int l = 0; l <= kMaxEvalDepth; ++l) { ape[l] = 0.0; sse[l] = 0.0; }
  Part py{0, 0, 0, 0, 0};
  for (int64_t r = lo + threadIdx.x; r < hi; r += blockDim.x) {
    const double yr = y[r];
    const double den = fmax(fabs(yr), 2.220446049250313e-16);
    const float* xr = X + r * d;
    uint32_t k = 0;
#pragma unroll
    for (int l = 0; l <= kMaxEvalDepth; ++l) {
      if (l <= depth) {
        const double e = yr - __ldg(value + k);
        ape[l] += __ddiv_rn(fabs(e), den);
        sse[l] += __dmul_rn(e, e);
        if (l < depth) k = step(nodes[k], xr);
      }
    }
    py.cnt += 1.0;
    const double delta = yr - py.mean;
    py.mean += __ddiv_rn(delta, py.cnt);
    py.m2 += __dmul_rn(delta, yr - py.mean);
  }
  // fixed-shape reduction: warp shuffles, then the 8 warps in order
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
  for (int l = 0; l <= kMaxEvalDepth; ++l) {
    if (l <= depth) {
      double a = ape[l], b = sse[l];
      for (int off = 16; off > 0; off >>= 1) {
        a += __shfl_down_sync(0xffffffffu, a, off);
        b += __shfl_down_sync(0xffffffffu, b, off);
      }
      if (lane == 0) { sh_ape[w][l] = a; sh_sse[w][l] = b; }
    }
  }
  py = block_reduce(py);
  if (threadIdx.x == 0) sh_y[0] = py;
  __syncthreads();
  if (threadIdx.x <= depth) {
    const int l = threadIdx.x;
    double a = 0.0, b = 0.0;
    for (int ww = 0; ww < (int)(blockDim.x >> 5); ++ww) { a += sh_ape[ww][l]; b += sh_sse[ww][l]; }
    DepthPart& o = parts[blockIdx.x];
    o.ape[l] = a;
    o.sse[l] = b;
    if (l == 0) {
      o.cnt = sh_y[0].cnt;
      o.mean = sh_y[0].mean;
      o.m2 = sh_y[0].m2;
    }
  }
}

__global__ void eval_depths_final_kernel(const DepthPart* __restrict__ parts, int nparts, int depth,
                                         int64_t n, int p_pred, double* __restrict__ out) {
  // thread l folds depth l in part order; thread 32 folds the y moments
  const int l = threadIdx.x;
  if (l <= depth) {
    double ape = 0.0, sse = 0.0;
    for (int i = 0; i < nparts; ++i) { ape += parts[i].ape[l]; sse += parts[i].sse[l]; }
    double na = 0, ma = 0, Ma = 0;
    for (int i = 0; i < nparts; ++i) chan_merge(na, ma, Ma, parts[i].cnt, parts[i].mean, parts[i].m2);
    const double nn = (double)n;
    double r2;
    if (Ma == 0.0) r2 = (sse == 0.0) ? 1.0 : 0.0;
    else r2 = 1.0 - sse / Ma;
    double adj;
    if (nn - (double)p_pred - 1.0 <= 0.0) adj = __longlong_as_double(0x7ff8000000000000ll);
    else adj = 1.0 - (1.0 - r2) * (nn - 1.0) / (nn - (double)p_pred - 1.0);
    out[3 * l] = ape / nn;
    out[3 * l + 1] = r2;
    out[3 * l + 2] = adj;
  }
}

// Feature importances (NEXT-1; Table III, "Gini coefficient" read as mean
// decrease in SSE, Reading R3): imp[f] = sum over internal nodes split on f of
// N*imp_P - N_L*imp_L - N_R*imp_R, normalised to sum 1.  One block, fixed order.
__global__ void __launch_bounds__(256) importances_kernel(const dt_node* __restrict__ nodes, int64_t count,
                                                          int d, double* __restrict__ imp) {
  __shared__ double sh[256];
  __shared__ double tot_sh;
  const int64_t per = (count + blockDim.x - 1) / blockDim.x;
  const int64_t k0 = threadIdx.x * per, k1 = min(count, k0 + per);
  for (int f = 0; f < d; ++f) {
    double acc = 0.0;
    for (int64_t k = k0; k < k1; ++k) {
      const dt_node a = nodes[k];
      if (a.feature != f) continue;
      const dt_node L = nodes[a.left], R = nodes[a.right];
      acc += (double)a.n_samples * a.impurity - (double)L.n_samples * L.impurity -
             (double)R.n_samples * R.impurity;
    }
    sh[threadIdx.x] = acc;
    __syncthreads();
    for (int off = 128; off > 0; off >>= 1) {
      if (threadIdx.x < off) sh[threadIdx.x] += sh[threadIdx.x + off];
      __syncthreads();
    }
    if (threadIdx.x == 0) imp[f] = sh[0];
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    double tot = 0.0;
    for (int f = 0; f < d; ++f) tot += imp[f];
    tot_sh = tot;
  }
  __syncthreads();
  if (tot_sh > 0.0)
    for (int f = threadIdx.x; f < d; f += blockDim.x) imp[f] = imp[f] / tot_sh;
}


// ------------------------------------------------------- factored DSE predict (NEXT-3) --

// The paper's design-space exploration estimates one CNN on n GPU configurations
// (T_est = t_dca + n * t_pm): candidate (i, j) = CNN row i composed with
// GPU row j, never materialised.  Tree features are re-encoded (0x80 | g = GPU column g,
// c = CNN column c).  Output-write bound at best: 8 B per prediction (the inputs are
// O(n_cnn + n_gpu)).
struct DseMap {
  uint8_t code[256];  // tree feature f -> 0x80 | GPU column, or CNN column
};

// GPU-specialised trees (the per-candidate cost of the factored DSE): for GPU row j the
// GPU-side decisions are fixed, so tree T_j = the tree with every GPU-feature node
// replaced by the child row j takes.  T_j keeps only CNN-feature nodes and leaves (C2
// tree, depth 20: ~220 of 11487 nodes, depth <= 13), and candidate (i, j) is a walk of
// T_j on CNN row i making the full walk's CNN-side comparisons in the same order, so the
// reached leaf (hence yhat) is identical.
//
// Rank form of the comparisons (4-byte nodes): per CNN column c, T_c = the thresholds
// RD32(t) of the tree's nodes on column c, sorted (duplicates kept); rank(t) = #{t' in
// T_c : t' < t} and r(x) = #{t' in T_c : t' < x}.  Then x > t <=> r(x) > rank(t) (if t < x
// every t' <= t is below x, so r(x) >= rank(t) + 1; if t >= x, r(x) <= rank(t)), NaN x
// has r = 0 (goes left, as x > t is false).  A T_j node is one word: rank << 20 | local
// left child a << 7 (right = a + 1; a * 128 is the child's byte offset in the interleaved
// layout) | CNN column * 4 (its byte offset in a rank row); leaves self-loop with rank 0xFFF
// (never exceeded: r(x) <= |T_c| <= kRankCap) and keep their full-tree id in a parallel
// word.  The 32 trees of a group of 32 consecutive GPU rows are interleaved (node k of
// lane j at word k * 32 + j), so a warp's node reads hit 32 distinct banks whatever nodes
// its lanes sit on: one shared-memory wavefront per node read, one per CNN rank read (the
// lanes read one row, pitch kRowPitch words).
constexpr int kSpecCap = 720;      // slots per T_j: 32 x 720 x (4 + 4) B = 180 KB of shared memory
constexpr int kRankCap = 4095;     // thresholds per CNN column in rank form (12-bit ranks)
constexpr int kSpecMaxCols = 32;   // CNN columns of the rank form
constexpr int kRowPitch = 33;      // words per staged CNN rank row (odd: conflict-free)
struct SpecMeta {
  int32_t P;      // padded T_j size of the group (max over its lanes), or -1: full-tree walks
  int32_t D;      // steps: max leaf depth of the group's T_j
};

// Block c: T_c (bitonic sort in shared memory, duplicates kept) and rank(t) of every tree
// node on column c (lower bound in T_c).
__global__ void __launch_bounds__(512) dse_rank_kernel(const uint2* __restrict__ gnodes, int count, DseMap map,
                                                       float* __restrict__ rt, uint32_t* __restrict__ rn,
                                                       uint16_t* __restrict__ nrank, int* __restrict__ bad) {
  __shared__ float th[4096];
  __shared__ uint32_t nk[kRankCap];
  __shared__ uint32_t s_n;
  const uint32_t c = blockIdx.x;
  if (threadIdx.x == 0) s_n = 0u;
  __syncthreads();
#pragma unroll 4
  for (int k = threadIdx.x; k < count; k += blockDim.x) {
    const uint2 nd = __ldg(gnodes + k);
    if ((nd.y & 0xFFFFFFu) == (uint32_t)k) continue;  // leaf
    if (map.code[nd.y >> 24] != c) continue;          // another column (or a GPU column)
    const uint32_t q = atomicAdd(&s_n, 1u);
    if (q < (uint32_t)kRankCap) {
      th[q] = __uint_as_float(nd.x);
      nk[q] = (uint32_t)k;
    }
  }
  __syncthreads();
  const uint32_t n = s_n;
  if (n > (uint32_t)kRankCap) {
    if (threadIdx.x == 0) *bad = 1;
    return;
  }
  uint32_t p2 = 1u;
  while (p2 < n) p2 <<= 1;
  for (uint32_t q = n + threadIdx.x; q < p2; q += blockDim.x) th[q] = INFINITY;  // thresholds are finite
  __syncthreads();
  for (uint32_t kk = 2; kk <= p2; kk <<= 1) {
    for (uint32_t jj = kk >> 1; jj > 0; jj >>= 1) {
      for (uint32_t i = threadIdx.x; i < p2; i += blockDim.x) {
        const uint32_t ixj = i ^ jj;
        if (ixj > i) {
          const float u = th[i], v = th[ixj];
          if ((u > v) == ((i & kk) == 0)) { th[i] = v; th[ixj] = u; }
        }
      }
      __syncthreads();
    }
  }
  for (uint32_t q = threadIdx.x; q < n; q += blockDim.x) rt[(size_t)c * kRankCap + q] = th[q];
  // rank of each collected node: lower bound of its threshold
  for (uint32_t q = threadIdx.x; q < n; q += blockDim.x) {
    const float t = __uint_as_float(__ldg(gnodes + nk[q]).x);
    uint32_t lo = 0u, hi = n;
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if (th[mid] < t) lo = mid + 1u;
      else hi = mid;
    }
    nrank[nk[q]] = (uint16_t)lo;
  }
  if (threadIdx.x == 0) rn[c] = n;
}

// r(x) of every CNN table entry (binary search in T_c); the tables are staged in shared
// memory, packed by column, when they fit (kSmemRanks floats), else searched in place.
constexpr int kSmemRanks = 12000;
__global__ void __launch_bounds__(1024) dse_cnn_rank_kernel(const float* __restrict__ cnn, int64_t total, int dc,
                                                            const float* __restrict__ rt,
                                                            const uint32_t* __restrict__ rn,
                                                            uint16_t* __restrict__ crank) {
  __shared__ float st[kSmemRanks];
  __shared__ uint32_t s_off[kSpecMaxCols + 1];
  const int ncols = min(dc, kSpecMaxCols);
  if (threadIdx.x == 0) {
    uint32_t o = 0;
    for (int c = 0; c < ncols; ++c) {
      s_off[c] = o;
      o += __ldg(rn + c);
    }
    s_off[ncols] = o;
  }
  __syncthreads();
  const bool smem = s_off[ncols] <= (uint32_t)kSmemRanks;
  if (smem) {
    for (int c = 0; c < ncols; ++c)
      for (uint32_t q = threadIdx.x; q < s_off[c + 1] - s_off[c]; q += blockDim.x)
        st[s_off[c] + q] = __ldg(rt + (size_t)c * kRankCap + q);
  }
  __syncthreads();
  const int64_t nrow = total / dc;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nrow; i += (int64_t)gridDim.x * blockDim.x) {
    for (int c = 0; c < dc; ++c) {  // a thread per row: no 64-bit division per entry
      const int64_t e = i * dc + c;
      const float x = __ldg(cnn + e);
      uint32_t lo = 0u, hi = 0u;  // first index with !(T < x)
      if (c < ncols) {
        hi = s_off[c + 1] - s_off[c];
        if (smem) {
          const float* T = st + s_off[c];
          while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (T[mid] < x) lo = mid + 1u;
            else hi = mid;
          }
        } else {
          const float* T = rt + (size_t)c * kRankCap;
          while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (__ldg(T + mid) < x) lo = mid + 1u;
            else hi = mid;
          }
        }
      }
      crank[e] = (uint16_t)lo;
    }
  }
}

// The specialiser reads the packed tree and the node ranks from shared memory when they
// fit (every DFS step is a dependent load), else from global memory.
template <bool kSmem>
struct SpecTree {
  const uint2* nodes;
  const uint16_t* rank;
  __device__ __forceinline__ uint2 node(uint32_t k) const { return kSmem ? nodes[k] : __ldg(nodes + k); }
  __device__ __forceinline__ uint32_t rk(uint32_t k) const { return kSmem ? rank[k] : __ldg(rank + k); }
};

template <bool kSmem>
__device__ __forceinline__ uint32_t dse_resolve(const SpecTree<kSmem>& tr, const DseMap& map,
                                                const float* __restrict__ grow, uint32_t k) {
  // follow GPU-feature nodes with row j's features (the full walk's comparison)
  for (;;) {
    const uint2 nd = tr.node(k);
    const uint32_t left = nd.y & 0xFFFFFFu;
    if (left == k) return k;  // leaf
    const uint32_t code = map.code[nd.y >> 24];
    if (!(code & 0x80u)) return k;  // CNN node
    k = (grow[code & 0x7Fu] > __uint_as_float(nd.x)) ? left + 1 : left;
  }
}

// Warp w of block g builds T_j (j = 32 g + w) breadth-first: the frontier of a level is
// the contiguous slot range [lo, hi) whose full-tree nodes sit in the slots' id words;
// each lane expands one frontier slot per round (an internal node's two children get
// consecutive slots, placed by a warp prefix sum; each child is resolved through the
// GPU-feature nodes with row j's features).  Returns the slots used (P), the deepest
// leaf (D) and whether the tree fits (slots, rank form).
template <bool kSmem>
__device__ void dse_spec_build(const SpecTree<kSmem>& tr, const DseMap& map, const float* __restrict__ grow,
                               bool live, bool ok, uint32_t* __restrict__ out, uint32_t& P, uint32_t& D) {
  const int lane = threadIdx.x & 31;
  const uint32_t lt = (1u << lane) - 1u;
  uint32_t* lid = out + (size_t)kSpecCap * 32;  // slot k of this tree: out[32 k], lid[32 k]
  P = 1u;
  D = 0u;
  if (!live || !ok) {  // padding row (its outputs are never written) or no rank form
    if (lane == 0) {
      out[0] = 0xFFF00000u;
      lid[0] = 0u;
    }
    return;
  }
  if (lane == 0) lid[0] = dse_resolve(tr, map, grow, 0u);
  __syncwarp();
  uint32_t lo = 0u, hi = 1u, depth = 0u;
  while (lo < hi) {
    uint32_t nfree = hi;  // the next level's slots follow this level's
    for (uint32_t base = lo; base < hi; base += 32u) {
      const uint32_t slot = base + (uint32_t)lane;
      const bool act = slot < hi;
      const uint32_t k = act ? lid[(size_t)slot * 32] : 0u;
      const uint2 nd = tr.node(k);
      const uint32_t left = nd.y & 0xFFFFFFu;
      const bool internal = act && left != k;
      const uint32_t code = map.code[nd.y >> 24];
      const uint32_t bal = __ballot_sync(0xffffffffu, internal);
      const bool bad = __any_sync(0xffffffffu, internal && code >= (uint32_t)kSpecMaxCols);
      if (bad || nfree + 2u * __popc(bal) > (uint32_t)kSpecCap) {
        P = 0xFFFFFFFFu;  // does not fit
        return;
      }
      if (internal) {
        const uint32_t ac = nfree + 2u * __popc(bal & lt);
        out[(size_t)slot * 32] = (tr.rk(k) << 20) | (ac << 7) | (code << 2);
        lid[(size_t)ac * 32] = dse_resolve(tr, map, grow, left);
        lid[(size_t)(ac + 1u) * 32] = dse_resolve(tr, map, grow, left + 1u);
      } else if (act) {
        out[(size_t)slot * 32] = 0xFFF00000u | (slot << 7);  // leaf: self-loop, rank never exceeded
        D = depth;
      }
      nfree += 2u * __popc(bal);
    }
    __syncwarp();  // the next level's id words are visible to the whole warp
    lo = hi;
    hi = nfree;
    ++depth;
  }
  P = hi;
  D = __reduce_max_sync(0xffffffffu, D);
}

// Block g (one warp per GPU row of the group): the packed tree, the node ranks and the
// group's GPU rows staged in shared memory (the tree when it fits), the 32 trees built,
// then the group's padded size and depth.
__global__ void __launch_bounds__(1024) dse_spec_kernel(const uint2* __restrict__ gnodes, int count, DseMap map,
                                                        const float* __restrict__ gpu, int64_t n_gpu, int dg,
                                                        const uint16_t* __restrict__ nrank, const int* __restrict__ bad,
                                                        bool smem_tree, uint32_t* __restrict__ spec,
                                                        SpecMeta* __restrict__ meta) {
  extern __shared__ __align__(16) unsigned char spec_smem[];
  __shared__ uint32_t s_p[32], s_d[32];
  const bool ok = *bad == 0;
  float* sg = reinterpret_cast<float*>(spec_smem);  // 32 x dg
  for (int e = threadIdx.x; e < 32 * dg; e += blockDim.x) {
    const int64_t jj = (int64_t)blockIdx.x * 32 + e / dg;
    sg[e] = jj < n_gpu ? __ldg(gpu + jj * dg + e % dg) : 0.f;
  }
  uint2* sn = reinterpret_cast<uint2*>(spec_smem + ((sizeof(float) * 32 * (size_t)dg + 15) & ~(size_t)15));
  uint16_t* sr = reinterpret_cast<uint16_t*>(sn + count);
  if (smem_tree) {
    for (int k = threadIdx.x; k < count; k += blockDim.x) {
      sn[k] = __ldg(gnodes + k);
      sr[k] = ok ? __ldg(nrank + k) : (uint16_t)0;
    }
  }
  __syncthreads();
  const int w = threadIdx.x >> 5;
  const bool live = (int64_t)blockIdx.x * 32 + w < n_gpu;
  uint32_t* out = spec + (size_t)blockIdx.x * kSpecCap * 64 + w;
  uint32_t P, D;
  if (smem_tree) dse_spec_build(SpecTree<true>{sn, sr}, map, sg + w * dg, live, ok, out, P, D);
  else dse_spec_build(SpecTree<false>{gnodes, nrank}, map, sg + w * dg, live, ok, out, P, D);
  if ((threadIdx.x & 31) == 0) {
    s_p[w] = ok ? P : 0xFFFFFFFFu;
    s_d[w] = D;
  }
  __syncthreads();
  if (threadIdx.x < 32) {
    const uint32_t p = __reduce_max_sync(0xffffffffu, s_p[threadIdx.x]);
    const uint32_t dd = __reduce_max_sync(0xffffffffu, s_d[threadIdx.x]);
    if (threadIdx.x == 0) meta[blockIdx.x] = SpecMeta{p <= (uint32_t)kSpecCap ? (int32_t)p : -1, (int32_t)dd};
  }
}

// Candidates (i, j): block = one group of 32 GPU rows (lane = j) x a range of CNN rows;
// each warp walks kR CNN rows at once (independent chains) on the group's trees in
// shared memory and writes yhat[i * n_gpu + j] for its 32 consecutive j (256 B per row).
// A group whose trees do not fit (meta P = -1) walks the full tree from global memory.
template <int kR>
__global__ void __launch_bounds__(1024, 1)
predict_dse_spec_kernel(const uint2* __restrict__ gnodes, const double* __restrict__ value, int depth, DseMap map,
                        const uint32_t* __restrict__ spec, const SpecMeta* __restrict__ meta, int ngroups,
                        const float* __restrict__ cnn, const uint16_t* __restrict__ crank, int64_t n_cnn, int dc,
                        const float* __restrict__ gpu, int64_t n_gpu, int dg, double* __restrict__ yhat) {
  extern __shared__ __align__(16) unsigned char dse_smem[];
  uint32_t* tn = reinterpret_cast<uint32_t*>(dse_smem);
  uint32_t* tl = tn + (size_t)kSpecCap * 32;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
  uint32_t* cs = tl + (size_t)kSpecCap * 32 + (size_t)w * kR * kRowPitch;
  const int g = (int)(blockIdx.x % (unsigned)ngroups);
  const int64_t part = blockIdx.x / (unsigned)ngroups, nparts = gridDim.x / (unsigned)ngroups;
  const SpecMeta mt = meta[g];
  const int64_t j = (int64_t)g * 32 + lane;
  const bool live = j < n_gpu;
  if (mt.P > 0) {
    const uint4* src = reinterpret_cast<const uint4*>(spec + (size_t)g * kSpecCap * 64);
    uint4* dst = reinterpret_cast<uint4*>(tn);
    const int n4 = mt.P * 8;  // P slots x 32 lanes x 4 B / 16 B
    for (int e = threadIdx.x; e < n4; e += blockDim.x) {
      dst[e] = __ldg(src + e);
      dst[kSpecCap * 8 + e] = __ldg(src + kSpecCap * 8 + e);
    }
  }
  __syncthreads();
  // this block's CNN rows: [r0, r1), in warp tiles of kR rows
  const int64_t per = (n_cnn + nparts - 1) / nparts;
  const int64_t r0 = part * per, r1 = min(n_cnn, r0 + per);
  const float* grow = gpu + (live ? j : 0) * dg;
  // shared byte addresses: my slot-0 word of the trees, my warp's rank rows.  The walk
  // loads are plain (schedulable) asm; these addresses pass through volatile movs placed
  // after the barriers that publish the data, so no load can be hoisted above them.
  uint32_t tn0, cs0;
  asm volatile("mov.u32 %0, %1;" : "=r"(tn0) : "r"((uint32_t)__cvta_generic_to_shared(tn) + 4u * lane));
  for (int64_t i0 = r0 + (int64_t)w * kR; i0 < r1; i0 += (int64_t)nwarps * kR) {
    double v[kR];
    if (mt.P > 0) {
      __syncwarp();
      for (int e = lane; e < kR * dc; e += 32) {
        const int r = e / dc, c = e - r * dc;
        cs[r * kRowPitch + c] = (i0 + r < r1) ? (uint32_t)__ldg(crank + (i0 + r) * dc + c) : 0u;
      }
      __syncwarp();
      asm volatile("mov.u32 %0, %1;" : "=r"(cs0) : "r"((uint32_t)__cvta_generic_to_shared(cs)));
      uint32_t ka[kR];  // shared byte address of my current node, per row
#pragma unroll
      for (int r = 0; r < kR; ++r) ka[r] = tn0;
      for (int l = 0; l < mt.D; ++l) {
#pragma unroll
        for (int r = 0; r < kR; ++r) {
          uint32_t nd, xr;
          asm("ld.shared.u32 %0, [%1];" : "=r"(nd) : "r"(ka[r]));
          asm("ld.shared.u32 %0, [%1];" : "=r"(xr) : "r"(cs0 + (uint32_t)(r * kRowPitch * 4) + (nd & 0x7Cu)));
          // child word: my slot-0 word + (a + go) * 128 B
          ka[r] = tn0 + (nd & 0xFFF80u) + (xr > (nd >> 20) ? 128u : 0u);
        }
      }
#pragma unroll
      for (int r = 0; r < kR; ++r) {
        uint32_t id;
        asm("ld.shared.u32 %0, [%1];" : "=r"(id) : "r"(ka[r] + (uint32_t)(kSpecCap * 32 * 4)));
        v[r] = __ldg(value + id);
      }
    } else {  // full tree, both tables from global memory
      uint32_t k[kR];
#pragma unroll
      for (int r = 0; r < kR; ++r) k[r] = 0;
      for (int l = 0; l < depth; ++l) {
#pragma unroll
        for (int r = 0; r < kR; ++r) {
          const uint2 nd = __ldg(gnodes + k[r]);
          const uint32_t code = map.code[nd.y >> 24], left = nd.y & 0xFFFFFFu;
          const int64_t ir = min(i0 + r, n_cnn - 1);
          const float x = (code & 0x80u) ? __ldg(grow + (code & 0x7Fu)) : __ldg(cnn + ir * dc + code);
          k[r] = (x > __uint_as_float(nd.x)) ? left + 1 : left;
        }
      }
#pragma unroll
      for (int r = 0; r < kR; ++r) v[r] = __ldg(value + k[r]);
    }
    if (live) {
#pragma unroll
      for (int r = 0; r < kR; ++r)
        if (i0 + r < r1) yhat[(i0 + r) * n_gpu + j] = v[r];
    }
  }
}

}  // namespace

dt_status predict_dse_impl(const dt_tree* t, const float* cnn, int64_t n_cnn, int32_t dc, const float* gpu,
                           int64_t n_gpu, int32_t dg, const int32_t* src, double* yhat, cudaStream_t s) {
  if (!t->dev_packed) return fail(DT_ERR_TOO_LARGE, "dt_predict_dse: tree has >= 2^24 nodes");
  DseMap map{};
  for (int f = 0; f < t->d; ++f) {
    if (src[f] >= 0) {
      if (src[f] >= dc) return fail(DT_ERR_INVALID_ARG, "dt_predict_dse: bad CNN column in feature_src");
      map.code[f] = (uint8_t)src[f];
    } else {
      const int g = -1 - src[f];
      if (g >= dg) return fail(DT_ERR_INVALID_ARG, "dt_predict_dse: bad GPU column in feature_src");
      map.code[f] = (uint8_t)(0x80 | g);
    }
  }
  if (n_cnn == 0 || n_gpu == 0) return DT_OK;
  // rank tables, the GPU-specialised trees of every group of 32 GPU rows (scratch from
  // the stream's pool, freed in stream order), then the candidates
  const int64_t ngroups = (n_gpu + 31) / 32;
  const int ncols = std::min<int>(dc, kSpecMaxCols);
  unsigned char* scratch = nullptr;
  const size_t b_spec = sizeof(uint32_t) * (size_t)kSpecCap * 64 * (size_t)ngroups;
  const size_t b_meta = sizeof(SpecMeta) * (size_t)ngroups;
  const size_t b_rt = sizeof(float) * (size_t)kRankCap * kSpecMaxCols;
  const size_t b_rn = sizeof(uint32_t) * kSpecMaxCols + 16;  // + the bad flag
  const size_t b_nr = ((sizeof(uint16_t) * (size_t)t->count) + 15) & ~(size_t)15;
  const size_t b_cr = sizeof(uint16_t) * (size_t)n_cnn * (size_t)dc;
  DT_CK(cudaMallocAsync((void**)&scratch, b_spec + b_meta + b_rt + b_rn + b_nr + b_cr, s));
  struct FreeScratch {  // stream-ordered release on every return path
    unsigned char* p;
    cudaStream_t s;
    ~FreeScratch() { cudaFreeAsync(p, s); }
  } free_scratch{scratch, s};
  uint32_t* spec = reinterpret_cast<uint32_t*>(scratch);
  SpecMeta* meta = reinterpret_cast<SpecMeta*>(scratch + b_spec);
  float* rt = reinterpret_cast<float*>(scratch + b_spec + b_meta);
  uint32_t* rn = reinterpret_cast<uint32_t*>(scratch + b_spec + b_meta + b_rt);
  int* bad = reinterpret_cast<int*>(rn + kSpecMaxCols);
  uint16_t* nrank = reinterpret_cast<uint16_t*>(scratch + b_spec + b_meta + b_rt + b_rn);
  uint16_t* crank = reinterpret_cast<uint16_t*>(scratch + b_spec + b_meta + b_rt + b_rn + b_nr);
  const int pr = prof_begin(PK_PREDICT, s, 4);
  DT_CK(cudaMemsetAsync(rn, 0, b_rn, s));
  if (dc > kSpecMaxCols) DT_CK(cudaMemsetAsync(bad, 0xff, sizeof(int), s));  // rank rows hold <= 32 columns
  if (ncols > 0)
    dse_rank_kernel<<<(unsigned)ncols, 512, 0, s>>>(t->dev_packed, (int)t->count, map, rt, rn, nrank, bad);
  DT_CK(cudaGetLastError());
  const int64_t total = n_cnn * (int64_t)dc;
  dse_cnn_rank_kernel<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>((n_cnn + 1023) / 1024, (int64_t)num_sms() * 2)), 1024, 0, s>>>(
      cnn, total, dc, rt, rn, crank);
  DT_CK(cudaGetLastError());
  const size_t g_sm = (sizeof(float) * 32 * (size_t)dg + 15) & ~(size_t)15;
  const size_t tree_sm = (sizeof(uint2) + sizeof(uint16_t)) * (size_t)t->count;
  const bool smem_tree = g_sm + tree_sm <= 200 * 1024;
  const size_t spec_sm = g_sm + (smem_tree ? tree_sm : 0);
  DT_CK(cudaFuncSetAttribute(dse_spec_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)spec_sm));
  dse_spec_kernel<<<(unsigned)ngroups, 1024, spec_sm, s>>>(t->dev_packed, (int)t->count, map, gpu, n_gpu, dg, nrank,
                                                         bad, smem_tree, spec, meta);
  DT_CK(cudaGetLastError());
  // kR CNN rows per warp: independent walks in flight
  constexpr int kR = 8, kThr = 1024;
  const size_t sm = sizeof(uint32_t) * (size_t)kSpecCap * 64 + sizeof(uint32_t) * (size_t)(kThr / 32) * kR * kRowPitch;
  auto kern = predict_dse_spec_kernel<kR>;
  DT_CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
  // blocks: every group x nparts row ranges, about 8 waves of the SMs
  int64_t nparts = std::max<int64_t>(1, (8 * (int64_t)num_sms() + ngroups - 1) / ngroups);
  nparts = std::min<int64_t>(nparts, std::max<int64_t>(1, (n_cnn + kR - 1) / kR));
  nparts = std::min<int64_t>(nparts, (int64_t)0x7fffffff / ngroups);
  kern<<<(unsigned)(ngroups * nparts), kThr, sm, s>>>(t->dev_packed, t->dev_value, t->depth, map, spec, meta,
                                                     (int)ngroups, cnn, crank, n_cnn, dc, gpu, n_gpu, dg, yhat);
  prof_end(pr, s, 8.0 * (double)n_cnn * (double)n_gpu);  // the yhat write (inputs are O(n_cnn + n_gpu))
  DT_CK(cudaGetLastError());
  return DT_OK;
}

dt_status importances_impl(const dt_tree* t, double* imp_host, cudaStream_t s) {
  dt_node* dn = nullptr;
  double* di = nullptr;
  DT_CK(cudaMallocAsync((void**)&dn, sizeof(dt_node) * (size_t)t->count, s));
  DT_CK(cudaMallocAsync((void**)&di, sizeof(double) * (size_t)t->d, s));
  DT_CK(cudaMemcpyAsync(dn, t->host, sizeof(dt_node) * (size_t)t->count, cudaMemcpyHostToDevice, s));
  const int pr = prof_begin(PK_EVAL, s, 1);
  importances_kernel<<<1, 256, 0, s>>>(dn, t->count, t->d, di);
  prof_end(pr, s, 48.0 * (double)t->count);
  DT_CK(cudaGetLastError());
  DT_CK(cudaMemcpyAsync(imp_host, di, sizeof(double) * (size_t)t->d, cudaMemcpyDeviceToHost, s));
  DT_CK(cudaFreeAsync(dn, s));
  DT_CK(cudaFreeAsync(di, s));
  DT_CK(cudaStreamSynchronize(s));
  return DT_OK;
}

dt_status eval_depths_impl(const dt_tree* t, const float* X, const double* y, int64_t n, int32_t p,
                           cudaStream_t s, double* out_host) {
  const int depth = t->depth;
  if (depth > kMaxEvalDepth) return fail(DT_ERR_TOO_LARGE, "dt_predict_eval_depths: tree depth > 32");
  if (!t->dev_packed) return fail(DT_ERR_TOO_LARGE, "dt_predict_eval_depths: tree has >= 2^24 nodes");
  int64_t chunk = 8192;
  int64_t nparts = (n + chunk - 1) / chunk;
  if (nparts > 2048) {
    nparts = 2048;
    chunk = (n + nparts - 1) / nparts;
    nparts = (n + chunk - 1) / chunk;
  }
  DepthPart* parts = nullptr;
  double* dout = nullptr;
  DT_CK(cudaMallocAsync((void**)&parts, sizeof(DepthPart) * (size_t)nparts, s));
  DT_CK(cudaMallocAsync((void**)&dout, sizeof(double) * 3 * (size_t)(depth + 1), s));
  const int pr = prof_begin(PK_EVAL, s, 2);
  eval_depths_partial_kernel<<<(unsigned)nparts, 256, 0, s>>>(t->dev_packed, t->dev_value, depth, X, t->d, y,
                                                              n, chunk, parts);
  eval_depths_final_kernel<<<1, 64, 0, s>>>(parts, (int)nparts, depth, n, p, dout);
  prof_end(pr, s, (4.0 * t->d + 8.0) * (double)n);
  DT_CK(cudaGetLastError());
  DT_CK(cudaMemcpyAsync(out_host, dout, sizeof(double) * 3 * (size_t)(depth + 1), cudaMemcpyDeviceToHost, s));
  DT_CK(cudaFreeAsync(parts, s));
  DT_CK(cudaFreeAsync(dout, s));
  DT_CK(cudaStreamSynchronize(s));
  return DT_OK;
}

// Wide-format traversal (trees of >= 2^24 nodes, see dt_internal.cuh): node k =
// {f32 bits of RD32(threshold), left, feature, 0}; leaves self-loop like the packed form.
__global__ void __launch_bounds__(256) predict_wide_kernel(const uint4* __restrict__ nodes,
                                                           const double* __restrict__ value, int depth,
                                                           const float* __restrict__ X, int64_t n, int d,
                                                           double* __restrict__ yhat) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
    const float* xr = X + r * d;
    uint32_t k = 0;
    for (int l = 0; l < depth; ++l) {
      const uint4 nd = __ldg(nodes + k);
      k = (__ldg(xr + nd.z) > __uint_as_float(nd.x)) ? nd.y + 1 : nd.y;
    }
    yhat[r] = __ldg(value + k);
  }
}

dt_status predict_impl(const dt_tree* t, const float* X, int64_t n, int32_t d, double* yhat,
                       cudaStream_t s) {
  const int pr = prof_begin(PK_PREDICT, s, 1);
  if (t->dev_wide) {
    const int64_t g = std::min<int64_t>((int64_t)num_sms() * 8, std::max<int64_t>(1, (n + 255) / 256));
    predict_wide_kernel<<<(unsigned)g, 256, 0, s>>>(t->dev_wide, t->dev_value, t->depth, X, n, d, yhat);
    DT_CK(cudaGetLastError());
    prof_end(pr, s, (4.0 * d + 8.0) * (double)n);
    return DT_OK;
  }
  const bool use_smem = t->count <= kMaxSmemNodes;
  const size_t smem = use_smem ? sizeof(uint2) * (size_t)t->count : 0;
  // carveout in percent of the 228 KB unified L1/smem: just what the tree needs
  const int carveout = use_smem ? (int)std::min<size_t>(100, (smem + 2048) * 100 / (228 * 1024) + 1) : 0;
  if (use_smem && (d == 16 || d == 32)) {
    // shared-memory column kernel: tree + one smem column per thread
    const int thr = (d == 16) ? 1024 : 512;
    const size_t sm = sizeof(uint2) * (size_t)t->count + sizeof(float) * (size_t)thr * d;
    if (sm <= 227 * 1024) {
      auto kern = (d == 16) ? predict_col_kernel<1024, 16, 1> : predict_col_kernel<512, 32, 1>;
      DT_CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
      int per_sm = 1;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, thr, sm);
      if (per_sm < 1) per_sm = 1;
      const int64_t g = std::min<int64_t>((int64_t)num_sms() * per_sm,
                                          std::max<int64_t>(1, (n + (int64_t)thr - 1) / (int64_t)thr));
      kern<<<(unsigned)g, thr, sm, s>>>(t->dev_packed, t->dev_value, (int)t->count, t->depth, X, n, yhat);
      DT_CK(cudaGetLastError());
      prof_end(pr, s, (4.0 * d + 8.0) * (double)n);
      return DT_OK;
    }
  }
  // generic: tree in shared memory when it fits, rows through L1
  dt_status st = use_smem ? launch_predict<true, 1024, 1>(t, X, n, d, yhat, s, carveout)
                          : launch_predict<false, 256, 4>(t, X, n, d, yhat, s, carveout);
  prof_end(pr, s, (4.0 * d + 8.0) * (double)n);  // row read + f64 written
  return st;
}

dt_status eval_impl(const double* y, const double* yhat, const float* X, const dt_tree* t,
                    int64_t n, int32_t p, cudaStream_t s, dt_metrics* out) {
  if (t && !t->dev_packed) {
    // wide tree (>= 2^24 nodes): predict into a scratch vector, then the plain metrics
    double* tmp = nullptr;
    DT_CK(cudaMallocAsync((void**)&tmp, sizeof(double) * (size_t)n, s));
    dt_status st = predict_impl(t, X, n, t->d, tmp, s);
    if (st == DT_OK) st = eval_impl(y, tmp, nullptr, nullptr, n, p, s, out);
    cudaFreeAsync(tmp, s);
    return st;
  }
  // Fixed partition of [0, n) into nparts chunks (deterministic for a given n); 1024 rows
  // per 256-thread block: 4 rows per thread, enough blocks to fill the SMs at 1M rows
  int64_t chunk = 1024;
  int64_t nparts = (n + chunk - 1) / chunk;
  if (nparts > 4096) {
    nparts = 4096;
    chunk = (n + nparts - 1) / nparts;
    nparts = (n + chunk - 1) / chunk;
  }
  Part* parts = nullptr;
  double* dout = nullptr;
  DT_CK(cudaMallocAsync(&parts, sizeof(Part) * (size_t)nparts, s));
  DT_CK(cudaMallocAsync(&dout, sizeof(double) * 3, s));
  const int pr = prof_begin(PK_EVAL, s, 2);
  if (t) {
    eval_partial_kernel<true><<<(unsigned)nparts, 256, 0, s>>>(
        y, nullptr, t->dev_packed, t->dev_value, t->depth, X, t->d, n, chunk, parts);
  } else {
    eval_partial_kernel<false><<<(unsigned)nparts, 256, 0, s>>>(y, yhat, nullptr, nullptr, 0,
                                                                nullptr, 0, n, chunk, parts);
  }
  DT_CK(cudaGetLastError());
  eval_final_kernel<<<1, 1024, 0, s>>>(parts, (int)nparts, n, p, dout);
  prof_end(pr, s, t ? (4.0 * t->d + 8.0) * (double)n : 16.0 * (double)n);
  DT_CK(cudaGetLastError());
  double h[3];
  DT_CK(cudaMemcpyAsync(h, dout, sizeof h, cudaMemcpyDeviceToHost, s));
  DT_CK(cudaFreeAsync(parts, s));
  DT_CK(cudaFreeAsync(dout, s));
  DT_CK(cudaStreamSynchronize(s));
  out->mape = h[0];
  out->r2 = h[1];
  out->adj_r2 = h[2];
  out->n = n;
  out->p = p;
  return DT_OK;
}

// dt_eval_sharded: each rank reduces its rows to one partial (sums + Welford moments),
// the partials are allgathered and merged in rank order (SURVEY 8e "Eval").
dt_status eval_sharded_impl(dt_comm* comm, const double* y, const double* yhat, int64_t n, int32_t p,
                            cudaStream_t s, dt_metrics* out) {
  const int world = comm_world(comm);
  int64_t chunk = 1024;  // the partition of eval_impl: one rank reproduces dt_eval bitwise
  int64_t nparts = n > 0 ? (n + chunk - 1) / chunk : 0;
  if (nparts > 4096) {
    nparts = 4096;
    chunk = (n + nparts - 1) / nparts;
    nparts = (n + chunk - 1) / chunk;
  }
  Part *parts = nullptr, *mine = nullptr, *all = nullptr;
  double* dout = nullptr;
  DT_CK(cudaMallocAsync(&parts, sizeof(Part) * (size_t)std::max<int64_t>(1, nparts), s));
  DT_CK(cudaMallocAsync(&mine, sizeof(Part), s));
  DT_CK(cudaMallocAsync(&all, sizeof(Part) * (size_t)world, s));
  DT_CK(cudaMallocAsync(&dout, sizeof(double) * 4, s));
  const int pr = prof_begin(PK_EVAL, s, 3);
  if (nparts > 0)
    eval_partial_kernel<false><<<(unsigned)nparts, 256, 0, s>>>(y, yhat, nullptr, nullptr, 0, nullptr, 0, n, chunk,
                                                                parts);
  eval_local_kernel<<<1, 1024, 0, s>>>(parts, (int)nparts, mine);
  DT_CK(cudaGetLastError());
  dt_status cst = comm_allgather(comm, mine, all, sizeof(Part), s);
  if (cst != DT_OK) return cst;
  eval_ranks_kernel<<<1, 32, 0, s>>>(all, world, p, dout);
  prof_end(pr, s, 16.0 * (double)n);
  DT_CK(cudaGetLastError());
  double h[4];
  DT_CK(cudaMemcpyAsync(h, dout, sizeof h, cudaMemcpyDeviceToHost, s));
  DT_CK(cudaFreeAsync(parts, s));
  DT_CK(cudaFreeAsync(mine, s));
  DT_CK(cudaFreeAsync(all, s));
  DT_CK(cudaFreeAsync(dout, s));
  DT_CK(cudaStreamSynchronize(s));
  out->mape = h[0];
  out->r2 = h[1];
  out->adj_r2 = h[2];
  out->n = (int64_t)h[3];
  out->p = p;
  return DT_OK;
}

}  // namespace dtl
