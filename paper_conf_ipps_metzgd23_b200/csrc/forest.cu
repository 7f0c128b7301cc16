// Random Forest = bagged CART ("the Random Forest Tree is
// an ensemble of Decision Trees", :231 "the decision is taken based on the average value
// of all included Decision Trees"; Readings R20, R21 in DESIGN.md).
//
// Fit: tree t is the exact CART of its bootstrap sample, n rows drawn with replacement by
// a counter-based SplitMix64 stream.  The table is presorted ONCE; each tree's level-0
// lists are the presorted lists with every entry repeated by its row's draw count (fit.cu
// forest_trees_impl, presort.cu forest_tree_enqueue), then dt_fit's level loop runs.
// Predict: one kernel, one row per thread, every tree walked in tree order (nodes
// through L1/L2), the fp64 sum divided by T -- HBM reads 4d B per row once.
#include <algorithm>
#include <mutex>
#include <vector>

#include "dt_internal.cuh"

struct dt_forest {
  std::vector<dt_tree*> trees;
  int32_t d = 0;
  int64_t split_evals = 0;
  const uint2** dev_nodes = nullptr;    // [T] packed node arrays (the trees' own copies)
  const double** dev_values = nullptr;  // [T]
  int32_t* dev_depth = nullptr;         // [T]
};

namespace dtl {

namespace {

// Reading R21: draw i of tree t.
__device__ __forceinline__ uint32_t boot_index(uint64_t seed, uint32_t t, uint64_t i, uint64_t n) {
  uint64_t z = seed + 0x9E3779B97F4A7C15ull * ((((uint64_t)t) << 32) + i + 1ull);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  z ^= z >> 31;
  return (uint32_t)(z % n);
}

__global__ void __launch_bounds__(256) boot_index_kernel(uint64_t seed, uint32_t t, int64_t n, uint32_t* idx) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    idx[i] = boot_index(seed, t, (uint64_t)i, (uint64_t)n);
}

__global__ void __launch_bounds__(256) forest_predict_kernel(const uint2* const* __restrict__ nodes,
                                                             const double* const* __restrict__ values,
                                                             const int32_t* __restrict__ depth, int T,
                                                             const float* __restrict__ X, int64_t n, int d,
                                                             double* __restrict__ yhat) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
    const float* xr = X + r * d;
    double acc = 0.0;
    for (int t = 0; t < T; ++t) {
      const uint2* nd = nodes[t];
      const int D = depth[t];
      uint32_t k = 0;
      for (int l = 0; l < D; ++l) {
        const uint2 q = __ldg(nd + k);
        const uint32_t f = q.y >> 24, left = q.y & 0xFFFFFFu;
        k = (__ldg(xr + f) > __uint_as_float(q.x)) ? left + 1 : left;  // Reading R5
      }
      acc = __dadd_rn(acc, __ldg(values[t] + k));  // tree order
    }
    yhat[r] = __ddiv_rn(acc, (double)T);
  }
}

}  // namespace

dt_status bootstrap_impl(uint64_t seed, int32_t t, int64_t n, uint32_t* idx, cudaStream_t s) {
  const int64_t g = std::min<int64_t>((n + 255) / 256, (int64_t)num_sms() * 8);
  boot_index_kernel<<<(unsigned)std::max<int64_t>(1, g), 256, 0, s>>>(seed, (uint32_t)t, n, idx);
  prof_add_launches(1);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

dt_status forest_fit_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t n_trees,
                          int32_t max_depth, int64_t min_leaf, uint64_t seed, cudaStream_t s, dt_forest** out) {
  dt_forest* fo = new dt_forest();
  fo->d = d;
  dt_status st = forest_trees_impl(X, y, n, d, n_trees, max_depth, min_leaf, seed, s, fo->trees);
  if (st != DT_OK) {
    dt_forest_free(fo);
    return st;
  }
  std::vector<const uint2*> hn(n_trees);
  std::vector<const double*> hv(n_trees);
  std::vector<int32_t> hd(n_trees);
  for (int32_t t = 0; t < n_trees; ++t) {
    fo->split_evals += fo->trees[t]->split_evals;
    if (!fo->trees[t]->dev_packed) {
      dt_forest_free(fo);
      return fail(DT_ERR_TOO_LARGE, "dt_forest_fit: a tree has >= 2^24 nodes (no packed predict form)");
    }
    hn[t] = fo->trees[t]->dev_packed;
    hv[t] = fo->trees[t]->dev_value;
    hd[t] = fo->trees[t]->depth;
  }
  cudaError_t e = cudaMalloc((void**)&fo->dev_nodes, sizeof(void*) * n_trees);
  if (e == cudaSuccess) e = cudaMalloc((void**)&fo->dev_values, sizeof(void*) * n_trees);
  if (e == cudaSuccess) e = cudaMalloc((void**)&fo->dev_depth, sizeof(int32_t) * n_trees);
  if (e == cudaSuccess) e = cudaMemcpyAsync(fo->dev_nodes, hn.data(), sizeof(void*) * n_trees, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(fo->dev_values, hv.data(), sizeof(void*) * n_trees, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(fo->dev_depth, hd.data(), sizeof(int32_t) * n_trees, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) {
    dt_forest_free(fo);
    return cuda_fail(e, "forest tables", __FILE__, __LINE__);
  }
  *out = fo;
  return DT_OK;
}

dt_status forest_predict_impl(const dt_forest* fo, const float* X, int64_t n, int32_t d, double* yhat,
                              cudaStream_t s) {
  const int64_t g = std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, (int64_t)num_sms() * 8));
  const int pr = prof_begin(PK_PREDICT, s, 1);
  forest_predict_kernel<<<(unsigned)g, 256, 0, s>>>(fo->dev_nodes, fo->dev_values, fo->dev_depth,
                                                    (int)fo->trees.size(), X, n, d, yhat);
  prof_end(pr, s, (4.0 * d + 8.0) * (double)n);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

}  // namespace dtl

extern "C" {

void dt_forest_free(dt_forest* fo) {
  if (!fo) return;
  for (dt_tree* t : fo->trees) dt_tree_free(t);
  if (fo->dev_nodes) cudaFree(fo->dev_nodes);
  if (fo->dev_values) cudaFree(fo->dev_values);
  if (fo->dev_depth) cudaFree(fo->dev_depth);
  delete fo;
}

int32_t dt_forest_num_trees(const dt_forest* fo) { return fo ? (int32_t)fo->trees.size() : 0; }

const dt_tree* dt_forest_tree(const dt_forest* fo, int32_t t) {
  if (!fo || t < 0 || t >= (int32_t)fo->trees.size()) return nullptr;
  return fo->trees[t];
}

int64_t dt_forest_split_evals(const dt_forest* fo) { return fo ? fo->split_evals : 0; }

}  // extern "C"
