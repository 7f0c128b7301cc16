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
// GPU row j, never materialised.  A CTA keeps the tree (features re-encoded: 0x80 | g =
// GPU column g, c = CNN column c), the transposed GPU table (thread j reads column
// entries j: conflict-free) and kR CNN rows in shared memory; thread j walks kR
// candidates (i0 + r, j) at once (independent chains) and writes yhat[(i0 + r) * n_gpu + j]
// (coalesced).  Output-write bound: 8 B per prediction (the inputs are O(n_cnn + n_gpu)).
struct DseMap {
  uint8_t code[256];  // tree feature f -> 0x80 | GPU column, or CNN column
};

template <bool kSmemTree, bool kSorted, int kR>
__global__ void __launch_bounds__(1024, 1)
predict_dse_kernel(const uint2* __restrict__ gnodes, const double* __restrict__ value, int count, int depth,
                   const float* __restrict__ cnn, int64_t n_cnn, int dc, const float* __restrict__ gpu,
                   int n_gpu, int dg, int p2, DseMap map, double* __restrict__ yhat) {
  extern __shared__ __align__(16) unsigned char dse_smem[];
  uint2* snodes = reinterpret_cast<uint2*>(dse_smem);
  float* gpu_t = reinterpret_cast<float*>(dse_smem + (kSmemTree ? sizeof(uint2) * (size_t)count : 0));
  float* cnn_s = gpu_t + (size_t)dg * n_gpu;
  // kSorted: sort keys (p2 >= n_gpu, a power of two), the GPU order, output staging
  unsigned long long* skey = reinterpret_cast<unsigned long long*>(
      reinterpret_cast<unsigned char*>(cnn_s) + ((sizeof(float) * kR * dc + 15) & ~(size_t)15));
  uint32_t* perm = reinterpret_cast<uint32_t*>(skey + (kSorted ? p2 : 0));
  double* out_s = reinterpret_cast<double*>(perm + (kSorted ? ((n_gpu + 3) & ~3) : 0));
  const int tid = threadIdx.x;
  auto recode = [&](uint2 nd) {
    nd.y = ((uint32_t)map.code[nd.y >> 24] << 24) | (nd.y & 0xFFFFFFu);
    return nd;
  };
  if (kSmemTree) {
    for (int k = tid; k < count; k += blockDim.x) snodes[k] = recode(gnodes[k]);
    __syncthreads();
  }
  if (kSorted) {
    // GPU rows grouped by the leaf they reach with CNN row 0: neighbouring threads then
    // share most of their GPU-side decisions for any CNN, so a warp's node reads hit
    // fewer distinct shared-memory words (broadcasts instead of bank conflicts).
    for (int j = tid; j < p2; j += blockDim.x) {
      unsigned long long key = ~0ull;
      if (j < n_gpu) {
        uint32_t k = 0;
        for (int l = 0; l < depth; ++l) {
          const uint2 nd = kSmemTree ? snodes[k] : recode(__ldg(gnodes + k));
          const uint32_t code = nd.y >> 24, left = nd.y & 0xFFFFFFu;
          const float x = (code & 0x80u) ? __ldg(gpu + (int64_t)j * dg + (code & 0x7Fu)) : __ldg(cnn + code);
          k = (x > __uint_as_float(nd.x)) ? left + 1 : left;
        }
        key = ((unsigned long long)k << 32) | (uint32_t)j;
      }
      skey[j] = key;
    }
    __syncthreads();
    for (int kk = 2; kk <= p2; kk <<= 1) {  // bitonic sort of (leaf, row)
      for (int jj = kk >> 1; jj > 0; jj >>= 1) {
        for (int i = tid; i < p2; i += blockDim.x) {
          const int ixj = i ^ jj;
          if (ixj > i) {
            const unsigned long long u = skey[i], v = skey[ixj];
            const bool up = (i & kk) == 0;
            if ((u > v) == up) { skey[i] = v; skey[ixj] = u; }
          }
        }
        __syncthreads();
      }
    }
    for (int j = tid; j < n_gpu; j += blockDim.x) perm[j] = (uint32_t)skey[j];
    __syncthreads();
  }
  for (int e = tid; e < dg * n_gpu; e += blockDim.x) {
    const int g = e / n_gpu, j = e - g * n_gpu;
    const int src = kSorted ? (int)perm[j] : j;
    gpu_t[e] = __ldg(gpu + (int64_t)src * dg + g);
  }
  const int64_t nblk = (n_cnn + kR - 1) / kR;
  for (int64_t b = blockIdx.x; b < nblk; b += gridDim.x) {
    const int64_t i0 = b * kR;
    __syncthreads();  // previous CNN rows consumed (and the tables above written)
    for (int e = tid; e < kR * dc; e += blockDim.x) {
      const int r = e / dc;
      cnn_s[e] = (i0 + r < n_cnn) ? __ldg(cnn + (i0 + r) * dc + (e - r * dc)) : 0.f;
    }
    __syncthreads();
    for (int j = tid; j < n_gpu; j += blockDim.x) {
      uint32_t k[kR];
#pragma unroll
      for (int r = 0; r < kR; ++r) k[r] = 0;
      for (int l = 0; l < depth; ++l) {
#pragma unroll
        for (int r = 0; r < kR; ++r) {
          const uint2 nd = kSmemTree ? snodes[k[r]] : recode(__ldg(gnodes + k[r]));
          const uint32_t code = nd.y >> 24, left = nd.y & 0xFFFFFFu;
          const float* src = (code & 0x80u) ? gpu_t + (code & 0x7Fu) * (uint32_t)n_gpu + j
                                            : cnn_s + r * dc + code;
          // go left iff !(x > RD32(t)) (Reading R5); leaves self-loop
          k[r] = (*src > __uint_as_float(nd.x)) ? left + 1 : left;
        }
      }
#pragma unroll
      for (int r = 0; r < kR; ++r) {
        if (kSorted) out_s[r * n_gpu + perm[j]] = __ldg(value + k[r]);
        else if (i0 + r < n_cnn) yhat[(i0 + r) * (int64_t)n_gpu + j] = __ldg(value + k[r]);
      }
    }
    if (kSorted) {  // the staged rows, in GPU order, coalesced
      __syncthreads();
      for (int e = tid; e < kR * n_gpu; e += blockDim.x) {
        const int r = e / n_gpu;
        if (i0 + r < n_cnn) yhat[i0 * (int64_t)n_gpu + e] = out_s[e];
      }
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
  // kR CNN rows per thread: independent tree walks in flight (measured 2 / 4 / 6 / 8 / 12 /
  // 16: 70 / 72 / 87 / 87 / 87 / 71 G predictions/s at 2^20 x 2^10)
  constexpr int kR = 8, kThr = 1024;
  const size_t cnn_bytes = (sizeof(float) * kR * (size_t)dc + 15) & ~(size_t)15;
  const size_t tables = sizeof(float) * (size_t)dg * (size_t)n_gpu + cnn_bytes;
  int p2 = 1;
  while (p2 < n_gpu) p2 <<= 1;
  const size_t sort_bytes = sizeof(unsigned long long) * (size_t)p2 + sizeof(uint32_t) * (size_t)((n_gpu + 3) & ~3) +
                            sizeof(double) * kR * (size_t)n_gpu;
  const size_t tree = sizeof(uint2) * (size_t)t->count;
  const size_t cap = 227 * 1024;
  if (tables > cap) return fail(DT_ERR_TOO_LARGE, "dt_predict_dse: GPU table too large for shared memory");
  const bool smem_tree = tree + tables <= cap;
  const bool sorted = (smem_tree ? tree : 0) + tables + sort_bytes <= cap;
  const size_t sm = (smem_tree ? tree : 0) + tables + (sorted ? sort_bytes : 0);
  auto kern = smem_tree ? (sorted ? predict_dse_kernel<true, true, kR> : predict_dse_kernel<true, false, kR>)
                        : (sorted ? predict_dse_kernel<false, true, kR> : predict_dse_kernel<false, false, kR>);
  DT_CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
  const int64_t nblk = (n_cnn + kR - 1) / kR;
  const int64_t g = std::min<int64_t>((int64_t)num_sms(), nblk);
  const int pr = prof_begin(PK_PREDICT, s, 1);
  kern<<<(unsigned)g, kThr, sm, s>>>(t->dev_packed, t->dev_value, (int)t->count, t->depth, cnn, n_cnn, dc, gpu,
                                     (int)n_gpu, dg, p2, map, yhat);
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
  // Fixed partition of [0, n) into nparts chunks (deterministic for a given n).
  int64_t chunk = 4096;
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
  int64_t chunk = 4096;
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
