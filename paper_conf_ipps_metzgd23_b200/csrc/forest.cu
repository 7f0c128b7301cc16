// Random Forest = bagged CART ("the Random Forest Tree is
// an ensemble of Decision Trees", :231 "the decision is taken based on the average value
// of all included Decision Trees"; Readings R20, R21 in DESIGN.md).
//
// Fit: tree t is the exact CART (dt_fit's whole B200 pipeline) of its bootstrap sample,
// n rows drawn with replacement by a counter-based SplitMix64 stream.  One gather kernel
// per tree writes the sample (rows in draw order) into a scratch table whose addresses do
// not change from tree to tree, so every tree after the first replays dt_fit's cached
// CUDA graph.  Predict: one kernel, one row per thread, every tree walked in tree order
// (nodes through L1/L2), the fp64 sum divided by T -- HBM reads 4d B per row once.
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

// Bootstrap sample of tree t: a warp per sample row, lanes over the row's features
// (coalesced 4d-byte row reads and writes).
__global__ void __launch_bounds__(256) boot_gather_kernel(uint64_t seed, uint32_t t, const float* __restrict__ X,
                                                          const double* __restrict__ y, int64_t n, int d,
                                                          float* __restrict__ Xb, double* __restrict__ yb) {
  const int lane = threadIdx.x & 31;
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = w0; i < n; i += nw) {
    const uint32_t r = boot_index(seed, t, (uint64_t)i, (uint64_t)n);  // same value in every lane
    for (int f = lane; f < d; f += 32) Xb[i * d + f] = __ldg(X + (int64_t)r * d + f);
    if (lane == 0) yb[i] = __ldg(y + r);
  }
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

namespace {
// The bootstrap scratch table outlives one dt_forest_fit: the next forest of the same
// shape gathers into the same addresses, so even its FIRST tree replays dt_fit's cached
// graph plan (with a fresh cudaMalloc per forest the addresses change, every forest
// re-captures and may evict another cached plan).  Measured: after the bench's DSE and
// grid sections a 16-tree forest took 105-1180 ms with per-call scratch, 66 ms alone.
// A second thread fitting a forest while the cache is in use gets a private table.
struct ForestScratch {
  std::mutex mu;
  float* X = nullptr;
  double* y = nullptr;
  int64_t n = 0;
  int32_t d = 0, device = -1;
};
ForestScratch g_scratch;

void scratch_free(ForestScratch& sc) {
  if (sc.X) cudaFree(sc.X);
  if (sc.y) cudaFree(sc.y);
  sc.X = nullptr;
  sc.y = nullptr;
  sc.n = 0;
  sc.d = 0;
  sc.device = -1;
}
}  // namespace

void forest_release_scratch() {
  std::lock_guard<std::mutex> lk(g_scratch.mu);
  scratch_free(g_scratch);
}

dt_status forest_fit_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t n_trees,
                          int32_t max_depth, int64_t min_leaf, uint64_t seed, cudaStream_t s, dt_forest** out) {
  dt_forest* fo = new dt_forest();
  fo->d = d;
  float* Xb = nullptr;
  double* yb = nullptr;
  std::unique_lock<std::mutex> lk(g_scratch.mu, std::try_to_lock);
  const bool cached = lk.owns_lock();
  auto cleanup = [&](dt_status st) {
    if (!cached) {
      if (Xb) cudaFree(Xb);
      if (yb) cudaFree(yb);
    }
    if (st != DT_OK) dt_forest_free(fo);
    return st;
  };
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return cleanup(cuda_fail(e, "cudaGetDevice", __FILE__, __LINE__));
  if (cached && g_scratch.X && g_scratch.n == n && g_scratch.d == d && g_scratch.device == dev) {
    Xb = g_scratch.X;
    yb = g_scratch.y;
  } else {
    if (cached) {
      e = cudaDeviceSynchronize();  // the previous scratch may still be read by a running fit
      if (e != cudaSuccess) return cleanup(cuda_fail(e, "cudaDeviceSynchronize", __FILE__, __LINE__));
      scratch_free(g_scratch);
    }
    e = cudaMalloc((void**)&Xb, sizeof(float) * (size_t)n * d);
    if (e == cudaSuccess) e = cudaMalloc((void**)&yb, sizeof(double) * (size_t)n);
    if (cached) {
      g_scratch.X = Xb;
      g_scratch.y = yb;
      g_scratch.n = n;
      g_scratch.d = d;
      g_scratch.device = dev;
      if (e != cudaSuccess) scratch_free(g_scratch);
    }
    if (e != cudaSuccess) {
      if (cached) Xb = nullptr, yb = nullptr;
      return cleanup(cuda_fail(e, "cudaMalloc (bootstrap sample)", __FILE__, __LINE__));
    }
  }
  const int64_t g = std::max<int64_t>(1, std::min<int64_t>((n + 7) / 8, (int64_t)num_sms() * 16));
  for (int32_t t = 0; t < n_trees; ++t) {
    boot_gather_kernel<<<(unsigned)g, 256, 0, s>>>(seed, (uint32_t)t, X, y, n, d, Xb, yb);
    prof_add_launches(1);
    e = cudaGetLastError();
    if (e != cudaSuccess) return cleanup(cuda_fail(e, "boot_gather_kernel", __FILE__, __LINE__));
    dt_tree* tr = nullptr;
    dt_status st = fit_impl(Xb, yb, n, d, max_depth, min_leaf, s, &tr);  // synchronises s
    if (st != DT_OK) return cleanup(st);
    fo->trees.push_back(tr);
    fo->split_evals += tr->split_evals;
  }
  std::vector<const uint2*> hn(n_trees);
  std::vector<const double*> hv(n_trees);
  std::vector<int32_t> hd(n_trees);
  for (int32_t t = 0; t < n_trees; ++t) {
    if (!fo->trees[t]->dev_packed)
      return cleanup(fail(DT_ERR_TOO_LARGE, "dt_forest_fit: a tree has >= 2^24 nodes (no packed predict form)"));
    hn[t] = fo->trees[t]->dev_packed;
    hv[t] = fo->trees[t]->dev_value;
    hd[t] = fo->trees[t]->depth;
  }
  e = cudaMalloc((void**)&fo->dev_nodes, sizeof(void*) * n_trees);
  if (e == cudaSuccess) e = cudaMalloc((void**)&fo->dev_values, sizeof(void*) * n_trees);
  if (e == cudaSuccess) e = cudaMalloc((void**)&fo->dev_depth, sizeof(int32_t) * n_trees);
  if (e == cudaSuccess) e = cudaMemcpyAsync(fo->dev_nodes, hn.data(), sizeof(void*) * n_trees, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(fo->dev_values, hv.data(), sizeof(void*) * n_trees, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(fo->dev_depth, hd.data(), sizeof(int32_t) * n_trees, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cleanup(cuda_fail(e, "forest tables", __FILE__, __LINE__));
  *out = fo;
  return cleanup(DT_OK);
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
