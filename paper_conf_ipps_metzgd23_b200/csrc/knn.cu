// KNN regression ("K-Nearest Neighbors ... non-linear
// dependencies", Table II :214; Reading R22 in DESIGN.md): yhat(q) = the mean target of
// the k training rows nearest to q by squared Euclidean distance, accumulated in fp64 by
// fused multiply-adds in feature order (acc = fma(q_f - x_f, q_f - x_f, acc)), ties to
// the lower training row.
//
// Brute force on the CUDA cores in fp64 (the exact distance of the definition; a GEMM
// expansion |q|^2 + |x|^2 - 2 q.x on the tensor cores rounds differently and would
// change the neighbour sets near ties).  kQ = 2 queries per thread (ILP and
// shared-memory reuse); the block streams the training set through shared memory in tiles of kTile
// rows (converted to f64 once per tile, read as warp-broadcasts); each thread keeps its
// queries' k best (distance, row) pairs sorted in registers.  Bound: the fp64 pipe, two
// instructions (DADD, DFMA) per (query, train row, feature).
#include <algorithm>

#include "dt_internal.cuh"

namespace dtl {

namespace {

constexpr int kKnnThreads = 128;
constexpr int kKnnTile = 64;  // training rows per shared-memory tile
constexpr int kKMaxAll = 16;

template <int D, int Q, int kKMax>
__global__ void __launch_bounds__(kKnnThreads)
knn_kernel(const float* __restrict__ Xtr, const double* __restrict__ ytr, int64_t ntr, const float* __restrict__ Xq,
           int64_t nq, int k, double* __restrict__ yhat) {
  __shared__ __align__(16) double tile[kKnnTile * D];
  const int64_t q0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * Q;
  double qv[Q][D];
#pragma unroll
  for (int a = 0; a < Q; ++a) {
    const int64_t q = min(q0 + a, nq - 1);
#pragma unroll
    for (int f = 0; f < D; ++f) qv[a][f] = (double)__ldg(Xq + q * D + f);
  }
  double bd[Q][kKMax];
  uint32_t bi[Q][kKMax];
  double worst[Q];
#pragma unroll
  for (int a = 0; a < Q; ++a) {
    worst[a] = INFINITY;
#pragma unroll
    for (int j = 0; j < kKMax; ++j) { bd[a][j] = INFINITY; bi[a][j] = 0u; }
  }
  for (int64_t t0 = 0; t0 < ntr; t0 += kKnnTile) {
    const int rows = (int)min((int64_t)kKnnTile, ntr - t0);
    __syncthreads();
    for (int e = threadIdx.x; e < rows * D; e += blockDim.x) tile[e] = (double)__ldg(Xtr + t0 * D + e);
    __syncthreads();
    for (int r = 0; r < rows; ++r) {
      const double2* xr = reinterpret_cast<const double2*>(tile + r * D);  // D even: 16-B aligned
      double acc[Q];
#pragma unroll
      for (int a = 0; a < Q; ++a) acc[a] = 0.0;
      if constexpr (D % 2 == 0) {
#pragma unroll
        for (int f2 = 0; f2 < D / 2; ++f2) {
          const double2 x = xr[f2];
#pragma unroll
          for (int a = 0; a < Q; ++a) {
            const double d0 = __dsub_rn(qv[a][2 * f2], x.x);
            acc[a] = __fma_rn(d0, d0, acc[a]);
            const double d1 = __dsub_rn(qv[a][2 * f2 + 1], x.y);
            acc[a] = __fma_rn(d1, d1, acc[a]);
          }
        }
      } else {
#pragma unroll
        for (int f = 0; f < D; ++f) {
          const double x = tile[r * D + f];
#pragma unroll
          for (int a = 0; a < Q; ++a) {
            const double df = __dsub_rn(qv[a][f], x);
            acc[a] = __fma_rn(df, df, acc[a]);
          }
        }
      }
#pragma unroll
      for (int a = 0; a < Q; ++a) {
        if (acc[a] < worst[a]) {  // strict: an equal distance keeps the earlier (lower) row
          const uint32_t row = (uint32_t)(t0 + r);
          bool placed = false;
#pragma unroll
          for (int j = kKMax - 1; j >= 0; --j) {
            if (j < k && !placed) {
              if (j > 0 && acc[a] < bd[a][j - 1]) {
                bd[a][j] = bd[a][j - 1];
                bi[a][j] = bi[a][j - 1];
              } else {
                bd[a][j] = acc[a];
                bi[a][j] = row;
                placed = true;
              }
            }
          }
#pragma unroll
          for (int j = 0; j < kKMax; ++j)
            if (j == k - 1) worst[a] = bd[a][j];
        }
      }
    }
  }
#pragma unroll
  for (int a = 0; a < Q; ++a) {
    if (q0 + a < nq) {
      double s = 0.0;
#pragma unroll
      for (int j = 0; j < kKMax; ++j)
        if (j < k) s = __dadd_rn(s, __ldg(ytr + bi[a][j]));
      yhat[q0 + a] = __ddiv_rn(s, (double)k);
    }
  }
}

// Two queries per thread (measured: 3 or 4 need > 200 registers and run ~2x slower);
// the k-best lists sized 8 when k <= 8 (the sklearn default k = 5), else 16.
template <int D>
void launch_knn(const float* Xtr, const double* ytr, int64_t ntr, const float* Xq, int64_t nq, int k, double* yhat,
                cudaStream_t s) {
  constexpr int Q = 2;
  const unsigned g = (unsigned)((nq + Q * kKnnThreads - 1) / (Q * kKnnThreads));
  if (k <= 8) knn_kernel<D, Q, 8><<<g, kKnnThreads, 0, s>>>(Xtr, ytr, ntr, Xq, nq, k, yhat);
  else knn_kernel<D, Q, 16><<<g, kKnnThreads, 0, s>>>(Xtr, ytr, ntr, Xq, nq, k, yhat);
}

}  // namespace

dt_status knn_impl(const float* Xtr, const double* ytr, int64_t ntr, int32_t d, const float* Xq, int64_t nq,
                   int32_t k, double* yhat, cudaStream_t s) {
  if (k > kKMaxAll) return fail(DT_ERR_TOO_LARGE, "dt_knn_predict: k must be <= 16");
  const int pr = prof_begin(PK_PREDICT, s, 1);
  switch (d) {  // the query row lives in registers: d is a compile-time constant
#define DT_KNN_CASE(D) \
  case D: launch_knn<D>(Xtr, ytr, ntr, Xq, nq, k, yhat, s); break;
    DT_KNN_CASE(1) DT_KNN_CASE(2) DT_KNN_CASE(3) DT_KNN_CASE(4) DT_KNN_CASE(5) DT_KNN_CASE(6)
    DT_KNN_CASE(7) DT_KNN_CASE(8) DT_KNN_CASE(10) DT_KNN_CASE(12) DT_KNN_CASE(16) DT_KNN_CASE(32)
#undef DT_KNN_CASE
    default:
      prof_end(pr, s, 0.0);
      return fail(DT_ERR_INVALID_ARG, "dt_knn_predict: d must be 1..8, 10, 12, 16 or 32");
  }
  prof_end(pr, s, 0.0);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

}  // namespace dtl
