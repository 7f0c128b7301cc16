// Batched tree prediction (the PM's estimate over DSE candidate sets, PAPER.md:205,
// :245-247) and the fused accuracy metrics (MAPE, R^2, adj-R^2; Table II
// :211-217).  HBM-bound: 4d B read + 8 B written per prediction; 16 B per metric element.
#include <math.h>

#include "dt_internal.cuh"

namespace dtl {

namespace {

constexpr int kPredThreads = 256;
constexpr int kRowsPerThread = 4;   // independent traversals per thread (ILP)
constexpr int kMaxSmemNodes = (227 * 1024) / 8;

// One traversal step: go left iff !(x > RD32(t)); for finite x this is exactly
// (double)x <= t (Reading R5).  Leaves self-loop (+inf threshold, left = self).
__device__ __forceinline__ uint32_t step(uint2 nd, const float* __restrict__ xr) {
  const uint32_t f = nd.y >> 24;
  const uint32_t left = nd.y & 0xFFFFFFu;
  const float x = __ldg(xr + f);
  return (x > __uint_as_float(nd.x)) ? left + 1 : left;
}

template <bool kSmem>
__global__ void __launch_bounds__(kPredThreads)
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

int pred_grid(int64_t n, size_t smem, bool use_smem) {
  int per_sm = 1;
  if (use_smem)
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, predict_kernel<true>, kPredThreads, smem);
  else
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, predict_kernel<false>, kPredThreads, 0);
  if (per_sm < 1) per_sm = 1;
  int64_t need = (n + (int64_t)kPredThreads * kRowsPerThread - 1) / ((int64_t)kPredThreads * kRowsPerThread);
  int64_t g = (int64_t)num_sms() * per_sm;
  return (int)(need < g ? (need < 1 ? 1 : need) : g);
}

}  // namespace

dt_status predict_impl(const dt_tree* t, const float* X, int64_t n, int32_t d, double* yhat,
                       cudaStream_t s) {
  const bool use_smem = t->count <= kMaxSmemNodes;
  const size_t smem = use_smem ? sizeof(uint2) * (size_t)t->count : 0;
  const int pr = prof_begin(PK_PREDICT, s, 1);
  if (use_smem) {
    DT_CK(cudaFuncSetAttribute(predict_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               (int)smem));
    predict_kernel<true><<<pred_grid(n, smem, true), kPredThreads, smem, s>>>(
        t->dev_packed, t->dev_value, (int)t->count, t->depth, X, n, d, yhat);
  } else {
    predict_kernel<false><<<pred_grid(n, 0, false), kPredThreads, 0, s>>>(
        t->dev_packed, t->dev_value, (int)t->count, t->depth, X, n, d, yhat);
  }
  prof_end(pr, s, (4.0 * d + 8.0) * (double)n);  // row read + f64 written
  DT_CK(cudaGetLastError());
  return DT_OK;
}

dt_status eval_impl(const double* y, const double* yhat, const float* X, const dt_tree* t,
                    int64_t n, int32_t p, cudaStream_t s, dt_metrics* out) {
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

}  // namespace dtl
