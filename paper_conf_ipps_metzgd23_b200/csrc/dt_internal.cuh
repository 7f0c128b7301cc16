// Internal declarations of libdt (B200 / sm_100a).  Not part of the C ABI.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/dt.h"

struct dt_tree {
  int64_t count = 0;          // number of nodes
  int32_t d = 0;              // features
  int32_t depth = 0;          // realised depth
  int64_t split_evals = 0;    // sum over searched nodes of N*d
  int32_t integer_mode = 0;
  dt_node* host = nullptr;    // count nodes, BFS
  // Device copy for prediction: packed 8-byte nodes {f32 thr (round-down), u32 f<<24|left}
  // (leaves self-loop: feature 0, thr +inf, left = self) plus f64 values.
  // Trees of >= kWideNodes nodes do not fit the 24-bit child field: they get the WIDE
  // form instead, 16-byte nodes {f32 bits of RD32(thr), left, feature, 0} (same
  // self-looping leaves), and dev_packed stays NULL (dt_predict / dt_predict_eval only).
  uint2* dev_packed = nullptr;
  uint4* dev_wide = nullptr;
  double* dev_value = nullptr;
  int device = -1;
  int async_alloc = 0;        // device arrays from cudaMallocAsync (dt_fit's pool)
};

constexpr int64_t kWideNodes = (int64_t)1 << 24;

namespace dtl {

// thread-local last error
void set_error(const std::string& msg);
dt_status fail(dt_status st, const std::string& msg);
dt_status cuda_fail(cudaError_t e, const char* what, const char* file, int line);

#define DT_CK(call)                                                          \
  do {                                                                       \
    cudaError_t e__ = (call);                                                \
    if (e__ != cudaSuccess) return dtl::cuda_fail(e__, #call, __FILE__, __LINE__); \
  } while (0)

// Build the device copy of a tree (packed nodes + values) from its host node array.
dt_status tree_upload(dt_tree* t, cudaStream_t s);

// Fit driver (fit.cu).
dt_status release_workspace_impl();
dt_status fit_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t max_depth,
                   int64_t min_leaf, cudaStream_t s, dt_tree** out);
dt_status forest_trees_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t n_trees, int32_t max_depth,
                            int64_t min_leaf, uint64_t seed, cudaStream_t s, std::vector<dt_tree*>& trees);
dt_status fit_grid_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t max_depth,
                        const int64_t* min_leafs, int32_t count, cudaStream_t s, dt_tree** outs);
dt_status fit_sharded_impl(dt_comm* comm, const float* X, const double* y, int64_t n_local, int64_t row_offset,
                           int64_t n_global, int32_t d, int32_t max_depth, int64_t min_leaf, cudaStream_t s,
                           dt_tree** out);
// Communicators (comm.cu).
int comm_rank(const dt_comm* c);
int comm_world(const dt_comm* c);
dt_status comm_allgather(dt_comm* c, const void* send, void* recv, size_t bytes, cudaStream_t s);
dt_status comm_allreduce_or_u32(dt_comm* c, uint32_t* buf, int64_t n, cudaStream_t s);
dt_status comm_allreduce_sum_u64(dt_comm* c, unsigned long long* buf, int64_t n, cudaStream_t s);
dt_status comm_alltoallv(dt_comm* c, const void* send, const size_t* scount, const size_t* sdispl, void* recv,
                         const size_t* rcount, const size_t* rdispl, cudaStream_t s);
// Predict / eval (predict.cu).
dt_status predict_dse_impl(const dt_tree* t, const float* cnn, int64_t n_cnn, int32_t dc, const float* gpu,
                           int64_t n_gpu, int32_t dg, const int32_t* src, double* yhat, cudaStream_t s);
dt_status predict_impl(const dt_tree* t, const float* X, int64_t n, int32_t d, double* yhat,
                       cudaStream_t s);
dt_status eval_impl(const double* y, const double* yhat, const float* X, const dt_tree* t,
                    int64_t n, int32_t p, cudaStream_t s, dt_metrics* out);
dt_status eval_sharded_impl(dt_comm* comm, const double* y, const double* yhat, int64_t n, int32_t p,
                            cudaStream_t s, dt_metrics* out);
dt_status importances_impl(const dt_tree* t, double* imp_host, cudaStream_t s);
dt_status eval_depths_impl(const dt_tree* t, const float* X, const double* y, int64_t n, int32_t p,
                           cudaStream_t s, double* out_host);
// Random forest (forest.cu).
dt_status bootstrap_impl(uint64_t seed, int32_t t, int64_t n, uint32_t* idx, cudaStream_t s);
dt_status forest_fit_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t n_trees,
                          int32_t max_depth, int64_t min_leaf, uint64_t seed, cudaStream_t s, dt_forest** out);
dt_status forest_predict_impl(const dt_forest* fo, const float* X, int64_t n, int32_t d, double* yhat,
                              cudaStream_t s);
// KNN regression (knn.cu).
dt_status knn_impl(const float* Xtr, const double* ytr, int64_t ntr, int32_t d, const float* Xq, int64_t nq,
                   int32_t k, double* yhat, cudaStream_t s);
// LOO (loo.cu).
dt_status loo_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t max_depth,
                   int64_t min_leaf, double* yhat, cudaStream_t s);
// Generators (gen.cu).
dt_status gen_table_impl(uint64_t seed, int64_t row0, int64_t n, int32_t d, int32_t real,
                         int32_t cbits, int32_t gbits, double unit_us, float* X, double* y,
                         cudaStream_t s);
dt_status gen_dse_impl(uint64_t seed, int64_t row0, int64_t n, int32_t gbits, float* X,
                       cudaStream_t s);

int num_sms();

// Profiling (prof.cu).  Kinds index the name table in prof.cu.
enum ProfKind {
  PK_PRESORT_KEYS = 0, PK_PRESORT_SORT, PK_PRESORT_BUILD, PK_ROOT, PK_SCAN, PK_SELECT,
  PK_NUMBER, PK_GOLEFT, PK_PARTITION, PK_PREDICT, PK_EVAL, PK_LOO, PK_GEN, PK_MEMSET
};
// Records an event before the launch(es) if profiling is on; counts `nlaunch` kernel
// launches of this library either way.  Returns a record index (or -1).
int prof_begin(int kind, cudaStream_t s, int nlaunch);
void prof_end(int idx, cudaStream_t s, double alg_bytes);
void prof_set_bytes(int idx, double alg_bytes);
bool prof_enabled();
// graph-captured profiling (dt_profile_enable(2)): event-record nodes of one fit graph
struct GRec {
  int kind;
  cudaEvent_t a, b;
  double bytes;
};
bool prof_graph_mode();
void prof_capture_target(std::vector<GRec>* v);  // prof_begin/end/set_bytes go to v (nullptr: off)
void prof_collect_graph(const std::vector<GRec>& v);  // after a replay completed
void prof_destroy_graph_recs(std::vector<GRec>& v);
void prof_add_launches(long long n);

}  // namespace dtl
