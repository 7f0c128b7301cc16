// C-ABI shim of libdt: argument validation, status codes, tree objects.
// Declarations and semantics: include/dt.h.
#include <math.h>
#include <stdio.h>
#include <string.h>

#include <cstdlib>
#include <string>
#include <vector>

#include "dt_internal.cuh"

namespace dtl {

static thread_local std::string g_err;

void set_error(const std::string& msg) { g_err = msg; }

dt_status fail(dt_status st, const std::string& msg) {
  g_err = msg;
  return st;
}

dt_status cuda_fail(cudaError_t e, const char* what, const char* file, int line) {
  char buf[512];
  snprintf(buf, sizeof buf, "CUDA error %d (%s) in %s at %s:%d", (int)e, cudaGetErrorString(e),
           what, file, line);
  g_err = buf;
  if (e == cudaErrorMemoryAllocation) return DT_ERR_OOM;
  return DT_ERR_CUDA;
}

int num_sms() {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return sms;
}

// Packed predict node: x = f32 bits of RD32(threshold) (x <= t  <=>  x <= RD32(t) for f32
// x, Reading R5), y = feature << 24 | left.  A leaf self-loops (feature 0, +inf, left =
// self) so every row runs exactly `depth` iterations without divergence on exit.
dt_status tree_upload(dt_tree* t, cudaStream_t s) {
  const bool wide = t->count >= kWideNodes;
  std::vector<uint2> packed(wide ? 0 : (size_t)t->count);
  std::vector<uint4> wnodes(wide ? (size_t)t->count : 0);
  std::vector<double> val((size_t)t->count);
  for (int64_t k = 0; k < t->count; ++k) {
    const dt_node& nd = t->host[k];
    val[(size_t)k] = nd.value;
    uint32_t bits, left, feat;
    if (nd.feature < 0) {
      float inf = INFINITY;
      memcpy(&bits, &inf, 4);
      left = (uint32_t)k;
      feat = 0;
    } else {
      // round-down of the fp64 threshold to f32
      float f = (float)nd.threshold;
      if ((double)f > nd.threshold) f = nextafterf(f, -INFINITY);
      memcpy(&bits, &f, 4);
      left = (uint32_t)nd.left;
      feat = (uint32_t)nd.feature;
    }
    if (wide) wnodes[(size_t)k] = make_uint4(bits, left, feat, 0u);
    else packed[(size_t)k] = make_uint2(bits, (feat << 24) | left);
  }
  DT_CK(cudaGetDevice(&t->device));
  if (wide) {
    DT_CK(cudaMalloc(&t->dev_wide, sizeof(uint4) * (size_t)t->count));
    DT_CK(cudaMemcpyAsync(t->dev_wide, wnodes.data(), sizeof(uint4) * (size_t)t->count, cudaMemcpyHostToDevice, s));
  } else {
    DT_CK(cudaMalloc(&t->dev_packed, sizeof(uint2) * (size_t)t->count));
    DT_CK(cudaMemcpyAsync(t->dev_packed, packed.data(), sizeof(uint2) * (size_t)t->count,
                          cudaMemcpyHostToDevice, s));
  }
  DT_CK(cudaMalloc(&t->dev_value, sizeof(double) * (size_t)t->count));
  DT_CK(cudaMemcpyAsync(t->dev_value, val.data(), sizeof(double) * (size_t)t->count,
                        cudaMemcpyHostToDevice, s));
  DT_CK(cudaStreamSynchronize(s));
  return DT_OK;
}

}  // namespace dtl

using namespace dtl;

static cudaStream_t S(void* p) { return (cudaStream_t)p; }

extern "C" {

const char* dt_last_error(void) { return g_err.c_str(); }

const char* dt_version(void) { return "libdt 0.1 sm_100a"; }

dt_status dt_fit(const float* X_dev, const double* y_dev, int64_t n, int32_t d,
                 int32_t max_depth, int64_t min_samples_leaf, void* stream, dt_tree** out) {
  if (!out) return fail(DT_ERR_INVALID_ARG, "dt_fit: out is NULL");
  *out = nullptr;
  if (!X_dev || !y_dev) return fail(DT_ERR_INVALID_ARG, "dt_fit: NULL X or y");
  if (n < 1) return fail(DT_ERR_INVALID_ARG, "dt_fit: n must be >= 1");
  if (n >= (int64_t)1 << 32) return fail(DT_ERR_TOO_LARGE, "dt_fit: n must be < 2^32");
  if (d < 1 || d > 255) return fail(DT_ERR_INVALID_ARG, "dt_fit: d must be in [1, 255]");
  if (max_depth < -1) return fail(DT_ERR_INVALID_ARG, "dt_fit: max_depth must be >= -1");
  if (min_samples_leaf < 1) return fail(DT_ERR_INVALID_ARG, "dt_fit: min_samples_leaf must be >= 1");
  return fit_impl(X_dev, y_dev, n, d, max_depth, min_samples_leaf, S(stream), out);
}

dt_status dt_fit_sharded(dt_comm* comm, const float* X_local_dev, const double* y_local_dev, int64_t n_local,
                         int64_t row_offset, int64_t n_global, int32_t d, int32_t max_depth, int64_t min_samples_leaf,
                         void* stream, dt_tree** out) {
  if (!out) return fail(DT_ERR_INVALID_ARG, "dt_fit_sharded: out is NULL");
  *out = nullptr;
  if (!comm) return fail(DT_ERR_INVALID_ARG, "dt_fit_sharded: comm is NULL");
  if (n_local < 0 || row_offset < 0) return fail(DT_ERR_INVALID_ARG, "dt_fit_sharded: n_local, row_offset must be >= 0");
  if (n_local > 0 && (!X_local_dev || !y_local_dev)) return fail(DT_ERR_INVALID_ARG, "dt_fit_sharded: NULL X or y");
  if (n_global < 1) return fail(DT_ERR_INVALID_ARG, "dt_fit_sharded: n_global must be >= 1");
  if (n_global >= (int64_t)1 << 32) return fail(DT_ERR_TOO_LARGE, "dt_fit_sharded: n_global must be < 2^32");
  if (row_offset + n_local > n_global) return fail(DT_ERR_INVALID_ARG, "dt_fit_sharded: row_offset + n_local > n_global");
  if (d < 1 || d > 255) return fail(DT_ERR_INVALID_ARG, "dt_fit_sharded: d must be in [1, 255]");
  if (max_depth < -1) return fail(DT_ERR_INVALID_ARG, "dt_fit_sharded: max_depth must be >= -1");
  if (min_samples_leaf < 1) return fail(DT_ERR_INVALID_ARG, "dt_fit_sharded: min_samples_leaf must be >= 1");
  return fit_sharded_impl(comm, X_local_dev, y_local_dev, n_local, row_offset, n_global, d, max_depth,
                          min_samples_leaf, S(stream), out);
}

dt_status dt_fit_grid(const float* X_dev, const double* y_dev, int64_t n, int32_t d, int32_t max_depth,
                      const int64_t* min_samples_leafs, int32_t count, void* stream, dt_tree** outs) {
  if (!outs || !min_samples_leafs || count < 1) return fail(DT_ERR_INVALID_ARG, "dt_fit_grid: need count >= 1 and arrays");
  for (int32_t i = 0; i < count; ++i) outs[i] = nullptr;
  if (!X_dev || !y_dev) return fail(DT_ERR_INVALID_ARG, "dt_fit_grid: NULL X or y");
  if (n < 1) return fail(DT_ERR_INVALID_ARG, "dt_fit_grid: n must be >= 1");
  if (n >= (int64_t)1 << 32) return fail(DT_ERR_TOO_LARGE, "dt_fit_grid: n must be < 2^32");
  if (d < 1 || d > 255) return fail(DT_ERR_INVALID_ARG, "dt_fit_grid: d must be in [1, 255]");
  if (max_depth < -1) return fail(DT_ERR_INVALID_ARG, "dt_fit_grid: max_depth must be >= -1");
  for (int32_t i = 0; i < count; ++i)
    if (min_samples_leafs[i] < 1) return fail(DT_ERR_INVALID_ARG, "dt_fit_grid: min_samples_leaf must be >= 1");
  dt_status st = fit_grid_impl(X_dev, y_dev, n, d, max_depth, min_samples_leafs, count, S(stream), outs);
  if (st != DT_OK) {
    for (int32_t i = 0; i < count; ++i) {
      dt_tree_free(outs[i]);
      outs[i] = nullptr;
    }
  }
  return st;
}

int64_t dt_tree_size(const dt_tree* t) { return t ? t->count : 0; }
const dt_node* dt_tree_nodes(const dt_tree* t) { return t ? t->host : nullptr; }
int32_t dt_tree_depth(const dt_tree* t) { return t ? t->depth : 0; }
int32_t dt_tree_num_features(const dt_tree* t) { return t ? t->d : 0; }
int64_t dt_tree_split_evals(const dt_tree* t) { return t ? t->split_evals : 0; }

dt_status dt_tree_from_nodes(const dt_node* nodes, int64_t count, int32_t d, dt_tree** out) {
  if (!out) return fail(DT_ERR_INVALID_ARG, "dt_tree_from_nodes: out is NULL");
  *out = nullptr;
  if (!nodes || count < 1) return fail(DT_ERR_INVALID_ARG, "dt_tree_from_nodes: empty");
  if (d < 1 || d > 255) return fail(DT_ERR_INVALID_ARG, "dt_tree_from_nodes: d must be in [1, 255]");
  if (count >= ((int64_t)1 << 31)) return fail(DT_ERR_TOO_LARGE, "dt_tree_from_nodes: >= 2^31 nodes");
  std::vector<int> refs((size_t)count, 0);
  int32_t depth = 0;
  if (nodes[0].depth != 0) return fail(DT_ERR_INVALID_ARG, "root depth != 0");
  for (int64_t k = 0; k < count; ++k) {
    const dt_node& a = nodes[k];
    if (!isfinite(a.value)) return fail(DT_ERR_NONFINITE, "non-finite node value");
    if (a.depth > depth) depth = a.depth;
    if (a.feature < 0) {
      if (a.left != -1 || a.right != -1) return fail(DT_ERR_INVALID_ARG, "leaf with children");
      continue;
    }
    if (a.feature >= d) return fail(DT_ERR_INVALID_ARG, "feature index >= d");
    if (!isfinite(a.threshold)) return fail(DT_ERR_NONFINITE, "non-finite threshold");
    if (a.left <= k || a.right != a.left + 1 || a.right >= count)
      return fail(DT_ERR_INVALID_ARG, "bad child links (need k < left, right == left + 1 < count)");
    if (nodes[a.left].depth != a.depth + 1 || nodes[a.right].depth != a.depth + 1)
      return fail(DT_ERR_INVALID_ARG, "child depth != parent depth + 1");
    refs[(size_t)a.left]++;
    refs[(size_t)a.right]++;
  }
  for (int64_t k = 1; k < count; ++k)
    if (refs[(size_t)k] != 1) return fail(DT_ERR_INVALID_ARG, "node not referenced exactly once");
  dt_tree* t = new dt_tree();
  t->count = count;
  t->d = d;
  t->depth = depth;
  t->host = (dt_node*)malloc(sizeof(dt_node) * (size_t)count);
  memcpy(t->host, nodes, sizeof(dt_node) * (size_t)count);
  dt_status st = tree_upload(t, 0);
  if (st != DT_OK) {
    dt_tree_free(t);
    return st;
  }
  *out = t;
  return DT_OK;
}

void dt_tree_free(dt_tree* t) {
  if (!t) return;
  // The device is synchronised first: an asynchronous predict still reading the nodes on
  // another (non-blocking) stream finishes before the memory can be reused.
  if (t->async_alloc) {
    cudaDeviceSynchronize();
    if (t->dev_packed) cudaFreeAsync(t->dev_packed, 0);
    if (t->dev_wide) cudaFreeAsync(t->dev_wide, 0);
    if (t->dev_value) cudaFreeAsync(t->dev_value, 0);
  } else {
    if (t->dev_packed) cudaFree(t->dev_packed);
    if (t->dev_wide) cudaFree(t->dev_wide);
    if (t->dev_value) cudaFree(t->dev_value);
  }
  free(t->host);
  delete t;
}

dt_status dt_predict(const dt_tree* t, const float* X_dev, int64_t n, int32_t d,
                     double* yhat_dev, void* stream) {
  if (!t) return fail(DT_ERR_INVALID_ARG, "dt_predict: tree is NULL");
  if (n < 0) return fail(DT_ERR_INVALID_ARG, "dt_predict: n < 0");
  if (n == 0) return DT_OK;
  if (!X_dev || !yhat_dev) return fail(DT_ERR_INVALID_ARG, "dt_predict: NULL X or yhat");
  if (d != t->d) return fail(DT_ERR_INVALID_ARG, "dt_predict: d differs from the tree's d");
  if (n >= ((int64_t)1 << 62)) return fail(DT_ERR_TOO_LARGE, "dt_predict: n >= 2^62");
  return predict_impl(t, X_dev, n, d, yhat_dev, S(stream));
}

dt_status dt_predict_dse(const dt_tree* t, const float* cnn_dev, int64_t n_cnn, int32_t dc,
                         const float* gpu_dev, int64_t n_gpu, int32_t dg, const int32_t* feature_src,
                         double* yhat_dev, void* stream) {
  if (!t) return fail(DT_ERR_INVALID_ARG, "dt_predict_dse: tree is NULL");
  if (n_cnn < 0 || n_gpu < 0) return fail(DT_ERR_INVALID_ARG, "dt_predict_dse: n_cnn, n_gpu must be >= 0");
  if (n_cnn == 0 || n_gpu == 0) return DT_OK;
  if (!cnn_dev || !gpu_dev || !yhat_dev || !feature_src)
    return fail(DT_ERR_INVALID_ARG, "dt_predict_dse: NULL pointer");
  if (dc < 1 || dg < 1 || dc > 128 || dg > 128) return fail(DT_ERR_INVALID_ARG, "dt_predict_dse: dc, dg in [1, 128]");
  if (n_gpu >= ((int64_t)1 << 24)) return fail(DT_ERR_TOO_LARGE, "dt_predict_dse: n_gpu >= 2^24");
  if (n_cnn >= ((int64_t)1 << 62) / n_gpu) return fail(DT_ERR_TOO_LARGE, "dt_predict_dse: n_cnn * n_gpu >= 2^62");
  return predict_dse_impl(t, cnn_dev, n_cnn, dc, gpu_dev, n_gpu, dg, feature_src, yhat_dev, S(stream));
}

dt_status dt_eval(const double* y_dev, const double* yhat_dev, int64_t n, int32_t p,
                  void* stream, dt_metrics* out) {
  if (!out) return fail(DT_ERR_INVALID_ARG, "dt_eval: out is NULL");
  if (!y_dev || !yhat_dev) return fail(DT_ERR_INVALID_ARG, "dt_eval: NULL y or yhat");
  if (n < 1) return fail(DT_ERR_INVALID_ARG, "dt_eval: n must be >= 1");
  if (p < 0) return fail(DT_ERR_INVALID_ARG, "dt_eval: p must be >= 0");
  return eval_impl(y_dev, yhat_dev, nullptr, nullptr, n, p, S(stream), out);
}

dt_status dt_predict_eval(const dt_tree* t, const float* X_dev, const double* y_dev, int64_t n,
                          int32_t d, int32_t p, void* stream, dt_metrics* out) {
  if (!out || !t) return fail(DT_ERR_INVALID_ARG, "dt_predict_eval: NULL tree or out");
  if (!X_dev || !y_dev) return fail(DT_ERR_INVALID_ARG, "dt_predict_eval: NULL X or y");
  if (n < 1) return fail(DT_ERR_INVALID_ARG, "dt_predict_eval: n must be >= 1");
  if (p < 0) return fail(DT_ERR_INVALID_ARG, "dt_predict_eval: p must be >= 0");
  if (d != t->d) return fail(DT_ERR_INVALID_ARG, "dt_predict_eval: d differs from the tree's d");
  return eval_impl(y_dev, nullptr, X_dev, t, n, p, S(stream), out);
}

dt_status dt_tree_truncate(const dt_tree* t, int32_t depth, dt_tree** out) {
  if (!out) return fail(DT_ERR_INVALID_ARG, "dt_tree_truncate: out is NULL");
  *out = nullptr;
  if (!t || depth < 0) return fail(DT_ERR_INVALID_ARG, "dt_tree_truncate: NULL tree or depth < 0");
  // BFS order: the nodes of depth <= D are a prefix-closed subset; renumber them in order.
  std::vector<int64_t> newid((size_t)t->count, -1);
  int64_t cnt = 0;
  for (int64_t k = 0; k < t->count; ++k)
    if (t->host[k].depth <= depth) newid[(size_t)k] = cnt++;
  std::vector<dt_node> nodes((size_t)cnt);
  for (int64_t k = 0; k < t->count; ++k) {
    if (newid[(size_t)k] < 0) continue;
    dt_node nd = t->host[k];
    if (nd.depth == depth || nd.feature < 0) {
      nd.feature = -1;
      nd.left = nd.right = -1;
      nd.threshold = 0.0;
    } else {
      nd.left = (int32_t)newid[(size_t)nd.left];
      nd.right = (int32_t)newid[(size_t)nd.right];
    }
    nodes[(size_t)newid[(size_t)k]] = nd;
  }
  dt_status st = dt_tree_from_nodes(nodes.data(), cnt, t->d, out);
  if (st == DT_OK) (*out)->split_evals = 0;
  return st;
}

dt_status dt_importances(const dt_tree* t, double* importances_host, void* stream) {
  if (!t || !importances_host) return fail(DT_ERR_INVALID_ARG, "dt_importances: NULL argument");
  return importances_impl(t, importances_host, S(stream));
}

dt_status dt_predict_eval_depths(const dt_tree* t, const float* X_dev, const double* y_dev, int64_t n,
                                 int32_t d, int32_t p, void* stream, double* metrics_host) {
  if (!t || !X_dev || !y_dev || !metrics_host) return fail(DT_ERR_INVALID_ARG, "dt_predict_eval_depths: NULL argument");
  if (n < 1) return fail(DT_ERR_INVALID_ARG, "dt_predict_eval_depths: n must be >= 1");
  if (p < 0) return fail(DT_ERR_INVALID_ARG, "dt_predict_eval_depths: p must be >= 0");
  if (d != t->d) return fail(DT_ERR_INVALID_ARG, "dt_predict_eval_depths: d differs from the tree's d");
  return eval_depths_impl(t, X_dev, y_dev, n, p, S(stream), metrics_host);
}

dt_status dt_loo(const float* X_dev, const double* y_dev, int64_t n, int32_t d, int32_t max_depth,
                 int64_t min_samples_leaf, double* yhat_oof_dev, void* stream) {
  if (!X_dev || !y_dev || !yhat_oof_dev) return fail(DT_ERR_INVALID_ARG, "dt_loo: NULL pointer");
  if (n < 2) return fail(DT_ERR_INVALID_ARG, "dt_loo: n must be >= 2");
  if (d < 1 || d > 255) return fail(DT_ERR_INVALID_ARG, "dt_loo: d must be in [1, 255]");
  if (max_depth < -1) return fail(DT_ERR_INVALID_ARG, "dt_loo: max_depth must be >= -1");
  if (min_samples_leaf < 1) return fail(DT_ERR_INVALID_ARG, "dt_loo: min_samples_leaf must be >= 1");
  if (n > 64 || d > 32) return fail(DT_ERR_TOO_LARGE, "dt_loo: needs n <= 64 and d <= 32");
  return loo_impl(X_dev, y_dev, n, d, max_depth, min_samples_leaf, yhat_oof_dev, S(stream));
}

dt_status dt_gen_table(uint64_t seed, int64_t row0, int64_t n, int32_t d, int32_t real,
                       int32_t cnn_pool_bits, int32_t gpu_pool_bits, double unit_us,
                       float* X_dev, double* y_dev, void* stream) {
  if (!X_dev) return fail(DT_ERR_INVALID_ARG, "dt_gen_table: X is NULL");
  if (n < 0 || row0 < 0) return fail(DT_ERR_INVALID_ARG, "dt_gen_table: n, row0 must be >= 0");
  if (d != 16 && d != 32) return fail(DT_ERR_INVALID_ARG, "dt_gen_table: d must be 16 or 32");
  if (cnn_pool_bits < 1 || cnn_pool_bits > 40 || gpu_pool_bits < 1 || gpu_pool_bits > 40)
    return fail(DT_ERR_INVALID_ARG, "dt_gen_table: pool bits must be in [1, 40]");
  if (!(unit_us > 0.0)) return fail(DT_ERR_INVALID_ARG, "dt_gen_table: unit_us must be > 0");
  if (n == 0) return DT_OK;
  return gen_table_impl(seed, row0, n, d, real, cnn_pool_bits, gpu_pool_bits, unit_us, X_dev,
                        y_dev, S(stream));
}

dt_status dt_gen_dse(uint64_t seed, int64_t row0, int64_t n, int32_t gpu_bits, float* X_dev,
                     void* stream) {
  if (!X_dev) return fail(DT_ERR_INVALID_ARG, "dt_gen_dse: X is NULL");
  if (n < 0 || row0 < 0) return fail(DT_ERR_INVALID_ARG, "dt_gen_dse: n, row0 must be >= 0");
  if (gpu_bits < 1 || gpu_bits > 40) return fail(DT_ERR_INVALID_ARG, "dt_gen_dse: gpu_bits in [1, 40]");
  if (n == 0) return DT_OK;
  return gen_dse_impl(seed, row0, n, gpu_bits, X_dev, S(stream));
}

dt_status dt_release_workspace(void) { return release_workspace_impl(); }

dt_status dt_bootstrap(uint64_t seed, int32_t tree, int64_t n, uint32_t* idx_dev, void* stream) {
  if (!idx_dev) return fail(DT_ERR_INVALID_ARG, "dt_bootstrap: idx is NULL");
  if (tree < 0) return fail(DT_ERR_INVALID_ARG, "dt_bootstrap: tree must be >= 0");
  if (n < 1) return fail(DT_ERR_INVALID_ARG, "dt_bootstrap: n must be >= 1");
  if (n >= (int64_t)1 << 32) return fail(DT_ERR_TOO_LARGE, "dt_bootstrap: n must be < 2^32");
  return bootstrap_impl(seed, tree, n, idx_dev, S(stream));
}

dt_status dt_forest_fit(const float* X_dev, const double* y_dev, int64_t n, int32_t d, int32_t n_trees,
                        int32_t max_depth, int64_t min_samples_leaf, uint64_t seed, void* stream,
                        dt_forest** out) {
  if (!out) return fail(DT_ERR_INVALID_ARG, "dt_forest_fit: out is NULL");
  *out = nullptr;
  if (!X_dev || !y_dev) return fail(DT_ERR_INVALID_ARG, "dt_forest_fit: NULL X or y");
  if (n < 1) return fail(DT_ERR_INVALID_ARG, "dt_forest_fit: n must be >= 1");
  if (d < 1 || d > 255) return fail(DT_ERR_INVALID_ARG, "dt_forest_fit: d must be in [1, 255]");
  if (n_trees < 1) return fail(DT_ERR_INVALID_ARG, "dt_forest_fit: n_trees must be >= 1");
  if (min_samples_leaf < 1) return fail(DT_ERR_INVALID_ARG, "dt_forest_fit: min_samples_leaf must be >= 1");
  if (max_depth < -1) return fail(DT_ERR_INVALID_ARG, "dt_forest_fit: max_depth must be >= -1");
  if (n >= (int64_t)1 << 32) return fail(DT_ERR_TOO_LARGE, "dt_forest_fit: n must be < 2^32");
  return forest_fit_impl(X_dev, y_dev, n, d, n_trees, max_depth, min_samples_leaf, seed, S(stream), out);
}

dt_status dt_forest_predict(const dt_forest* forest, const float* X_dev, int64_t n, int32_t d,
                            double* yhat_dev, void* stream) {
  if (!forest) return fail(DT_ERR_INVALID_ARG, "dt_forest_predict: forest is NULL");
  if (n < 0) return fail(DT_ERR_INVALID_ARG, "dt_forest_predict: n < 0");
  if (n == 0) return DT_OK;
  if (!X_dev || !yhat_dev) return fail(DT_ERR_INVALID_ARG, "dt_forest_predict: NULL X or yhat");
  if (d != dt_tree_num_features(dt_forest_tree(forest, 0)))
    return fail(DT_ERR_INVALID_ARG, "dt_forest_predict: d differs from the forest's d");
  return forest_predict_impl(forest, X_dev, n, d, yhat_dev, S(stream));
}

dt_status dt_knn_predict(const float* Xtr_dev, const double* ytr_dev, int64_t n_train, int32_t d,
                         const float* Xq_dev, int64_t n_query, int32_t k, double* yhat_dev, void* stream) {
  if (!Xtr_dev || !ytr_dev) return fail(DT_ERR_INVALID_ARG, "dt_knn_predict: NULL training data");
  if (n_train < 1) return fail(DT_ERR_INVALID_ARG, "dt_knn_predict: n_train must be >= 1");
  if (n_train >= (int64_t)1 << 32) return fail(DT_ERR_TOO_LARGE, "dt_knn_predict: n_train must be < 2^32");
  if (k < 1 || k > n_train) return fail(DT_ERR_INVALID_ARG, "dt_knn_predict: need 1 <= k <= n_train");
  if (n_query < 0) return fail(DT_ERR_INVALID_ARG, "dt_knn_predict: n_query < 0");
  if (n_query == 0) return DT_OK;
  if (!Xq_dev || !yhat_dev) return fail(DT_ERR_INVALID_ARG, "dt_knn_predict: NULL queries or yhat");
  return knn_impl(Xtr_dev, ytr_dev, n_train, d, Xq_dev, n_query, k, yhat_dev, S(stream));
}

dt_status dt_eval_sharded(dt_comm* comm, const double* y_dev, const double* yhat_dev, int64_t n_local, int32_t p,
                          void* stream, dt_metrics* out) {
  if (!comm) return fail(DT_ERR_INVALID_ARG, "dt_eval_sharded: comm is NULL");
  if (!out) return fail(DT_ERR_INVALID_ARG, "dt_eval_sharded: out is NULL");
  if (n_local < 0) return fail(DT_ERR_INVALID_ARG, "dt_eval_sharded: n_local < 0");
  if (n_local > 0 && (!y_dev || !yhat_dev)) return fail(DT_ERR_INVALID_ARG, "dt_eval_sharded: NULL y or yhat");
  if (p < 0) return fail(DT_ERR_INVALID_ARG, "dt_eval_sharded: p must be >= 0");
  return eval_sharded_impl(comm, y_dev, yhat_dev, n_local, p, S(stream), out);
}

}  // extern "C"
