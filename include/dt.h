/*
 * include/dt.h -- C ABI of the B200-native CART hot path (libdt.so).
 *
 * The operations are those of the paper's predictive model (PM): a Decision-Tree
 * regressor trained on rows d = (y, p, c_1..c_m, t) (Eq. 1; "Decision
 * Tree regression"), used to estimate performance for many
 * (CNN, GPU) candidates in a design-space exploration (T_est = t_dca + n*t_pm,
 * PAPER.md:245-247), and judged by MAPE, R^2 and adjusted R^2 (Table II
 * :211-217).  The paper fixes no hyper-parameter, tie rule or threshold rule; the
 * readings used here are listed in DESIGN.md ("Readings", R1-R24).  Beyond the tree, the
 * library carries the paper's other non-linear models (Random Forest as bagged CART,
 * KNN regression), a factored DSE predictor and row / feature sharded
 * multi-GPU calls.
 *
 * Conventions (all calls):
 *  - Every call returns dt_status; DT_OK == 0.  On error, dt_last_error() returns a
 *    thread-local message.  Arguments are validated before any launch.
 *  - *_dev arguments are CUDA device pointers owned by the caller (e.g. torch tensors);
 *    the library never frees caller memory.  *_host arguments are host pointers.
 *  - X is n x d float32 ROW-MAJOR (row r, feature f at X[r*d + f]); y and yhat are
 *    float64.  1 <= d <= 255.  Non-finite X or y -> DT_ERR_NONFINITE.
 *  - `stream` is a cudaStream_t (0 = legacy default stream).  Calls documented "async"
 *    enqueue work and return; calls documented "sync" synchronise `stream` first.
 *  - A sticky CUDA error returns DT_ERR_CUDA; the process must then re-initialise.
 *  - Distinct dt_tree objects are independent and may be used from different threads.
 */
#ifndef DT_H_
#define DT_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  DT_OK = 0,
  DT_ERR_INVALID_ARG = 1,
  DT_ERR_NONFINITE = 2,
  DT_ERR_OOM = 3,
  DT_ERR_CUDA = 4,
  DT_ERR_NCCL = 5,
  DT_ERR_TOO_LARGE = 6
} dt_status;

/* One tree node, 48 bytes, nodes in BFS order (node 0 = root; a level's nodes in index
 * order; a split appends left then right, so right == left + 1) -- Reading R9. */
typedef struct {
  int32_t feature;   /* split feature, -1 for a leaf                                    */
  int32_t left;      /* left child index, -1 for a leaf                                 */
  int32_t right;     /* right child index (== left + 1), -1 for a leaf                  */
  int32_t depth;     /* root = 0                                                        */
  double threshold;  /* go left iff (double)x[feature] <= threshold; 0.0 for leaves     */
  double value;      /* mean of y over the node's training rows (every node)            */
  double impurity;   /* SSE / n_samples of the node's training rows                     */
  int64_t n_samples; /* training rows in the node                                       */
} dt_node;

typedef struct dt_tree dt_tree; /* opaque: owns a host copy and a device copy of the nodes */

/* Accuracy metrics of Table II.  mape is a fraction (x100 for %),
 * MAPE = mean |y - yhat| / max(|y|, DBL_EPSILON) (Reading R12); r2 = 1 - SSE/SST,
 * unclamped, with r2 = (SSE == 0 ? 1 : 0) when SST == 0 (R13); adj_r2 =
 * 1 - (1 - r2)(n - 1)/(n - p - 1), NaN when n - p - 1 <= 0 (R14). */
typedef struct {
  double mape;
  double r2;
  double adj_r2;
  int64_t n;
  int32_t p;
} dt_metrics;

/* ------------------------------------------------------------------ fit ----------- */

/* dt_fit -- greedy CART regression (squared-error / variance reduction), exhaustive over
 * every feature and every threshold at every node (Readings R1-R10).
 *   X_dev  n x d f32 row-major, y_dev n f64 (device).  1 <= n < 2^32.
 *   max_depth: -1 = unlimited, 0 = a single root leaf.
 *   min_samples_leaf >= 1 (min_samples_split is 2 * min_samples_leaf, R2).
 * Split rule: for feature f and the node's rows ordered by (x_f, row id), position i
 * (first i rows left) is valid iff x[i-1] < x[i] and both children keep >=
 * min_samples_leaf rows; the gain (S'_L n_R - S'_R n_L)^2 / (N n_L n_R) of the
 * per-node-centered sums is maximised; ties go to the lowest feature, then the lowest
 * threshold; threshold = x[i-1]/2 + x[i]/2 in fp64 (R4, R5, R19).  A node is a leaf if
 * depth == max_depth, N < 2*min_samples_leaf, all its y are equal, or no position is
 * valid (R8).
 * Storage: integral targets with |y| < 2^31 travel through the level lists as int32
 * (R24); every sum and gain is still the same f64 value.  Repeated bounded-depth fits
 * (max_depth <= 24) of the same shape replay a cached CUDA graph (dt_release_workspace).
 * Sync: returns once the tree is complete; *out is owned by the caller (dt_tree_free).
 * Errors: INVALID_ARG (n, d, max_depth, min_samples_leaf, null pointers), NONFINITE,
 * TOO_LARGE (n >= 2^32 or workspace beyond device memory), OOM, CUDA. */
dt_status dt_fit(const float* X_dev, const double* y_dev, int64_t n, int32_t d,
                 int32_t max_depth, int64_t min_samples_leaf, void* stream, dt_tree** out);

/* dt_fit_grid -- the trees of dt_fit(X, y, n, d, max_depth, m) for every m in
 * min_samples_leafs[0 .. count) (BASELINE configs[4]'s (max_depth x min_samples_leaf)
 * grid; the depths come from dt_tree_truncate / dt_predict_eval_depths): ONE presort of the
 * table, then one level loop per m from a snapshot of the presorted lists (a greedy tree
 * depends on m only through its leaf rules).  outs[i] receives tree i (owned by the
 * caller; all NULL on error).  Needs ~16 B per (row, feature) beyond dt_fit's workspace.
 * Sync.  Errors as dt_fit. */
dt_status dt_fit_grid(const float* X_dev, const double* y_dev, int64_t n, int32_t d, int32_t max_depth,
                      const int64_t* min_samples_leafs, int32_t count, void* stream, dt_tree** outs);

/* Number of nodes; host view of the node array (valid until dt_tree_free). */
int64_t dt_tree_size(const dt_tree* tree);
const dt_node* dt_tree_nodes(const dt_tree* tree);
/* Realised depth (max node depth), the number of features the tree was fitted on, and
 * the split-eval count of the fit that produced it: sum over searched nodes (nodes not
 * made leaves by the depth / size / purity rules) of N*d -- the numerator of the
 * headline metric "row.feature split evals/s" (BASELINE.json).  Trees made
 * by dt_tree_from_nodes report 0 split evals. */
int32_t dt_tree_depth(const dt_tree* tree);
int32_t dt_tree_num_features(const dt_tree* tree);
int64_t dt_tree_split_evals(const dt_tree* tree);

/* Build a tree from a caller-supplied node array (e.g. a saved model or the oracle's
 * output).  Validates BFS links (right == left + 1, children after parent, depth =
 * parent depth + 1, every non-root node referenced once), 0 <= feature < d for internal
 * nodes, finite thresholds and values.  Copies the nodes; sync. */
dt_status dt_tree_from_nodes(const dt_node* nodes_host, int64_t count, int32_t d,
                             dt_tree** out);
void dt_tree_free(dt_tree* tree);

/* ------------------------------------------------------------------ predict ------- */

/* dt_predict -- the PM's estimate for every candidate row: from the
 * root go left iff (double)x[feature] <= threshold until a leaf; yhat = leaf value.
 * X_dev n x d f32 row-major (d must equal the tree's d), yhat_dev n f64.  n >= 0 (n == 0
 * is a no-op), n < 2^62.  Async on stream. */
dt_status dt_predict(const dt_tree* tree, const float* X_dev, int64_t n, int32_t d,
                     double* yhat_dev, void* stream);

/* dt_predict_dse -- factored design-space exploration (the PM
 * estimates ONE CNN on n candidate GPUs, T_est = t_dca + n * t_pm):
 * the candidates are the cross product of a CNN table and a GPU table, never
 * materialised.  cnn_dev: n_cnn x dc f32 row-major (the CNN-side features of each CNN);
 * gpu_dev: n_gpu x dg f32 row-major (the GPU-side features of each configuration).
 * feature_src (HOST, dt_tree_num_features(tree) entries) says where tree feature f comes
 * from: c >= 0 -> CNN column c, -1 - g -> GPU column g.  Candidate (i, j) is the row
 * x[f] = feature_src[f] >= 0 ? cnn[i][feature_src[f]] : gpu[j][-1 - feature_src[f]], and
 * yhat_dev[i * n_gpu + j] (f64, n_cnn * n_gpu entries, CNN-major) is exactly what
 * dt_predict returns for that row.  1 <= dc, dg <= 128; n_gpu < 2^24.  Method: per group
 * of 32 GPU rows the tree is specialised (GPU-feature nodes resolved, CNN thresholds in
 * rank form) into shared memory and each candidate walks only CNN-side decisions; groups
 * whose specialised trees exceed 720 nodes, trees with > 4095 thresholds on one CNN
 * column, and dc > 32 fall back to full-tree walks (same results).
 * Scratch: ~184 KB per GPU group + 2 B per CNN table entry, from the stream-ordered pool.
 * Errors: INVALID_ARG (NULL pointers, bad feature_src), TOO_LARGE.  Async on stream. */
dt_status dt_predict_dse(const dt_tree* tree, const float* cnn_dev, int64_t n_cnn, int32_t dc,
                         const float* gpu_dev, int64_t n_gpu, int32_t dg,
                         const int32_t* feature_src, double* yhat_dev, void* stream);

/* ------------------------------------------------------------------ eval ---------- */

/* dt_eval -- MAPE, R^2, adjusted R^2 of yhat against y (Table II).
 * n >= 1, p >= 0 (number of predictors for adj-R^2).  Sync: returns the metrics in *out. */
dt_status dt_eval(const double* y_dev, const double* yhat_dev, int64_t n, int32_t p,
                  void* stream, dt_metrics* out);

/* dt_predict_eval -- held-out evaluation fused into prediction (no yhat round trip):
 * metrics of dt_predict(tree, X) against y.  Sync. */
dt_status dt_predict_eval(const dt_tree* tree, const float* X_dev, const double* y_dev,
                          int64_t n, int32_t d, int32_t p, void* stream, dt_metrics* out);

/* dt_tree_truncate -- the tree cut at `depth` (nodes of depth == depth become leaves,
 * keeping their values).  Greedy CART is prefix-consistent: dt_fit(X, y, D', m) equals
 * dt_tree_truncate(dt_fit(X, y, D, m), D') for D' <= D (tests), which turns a
 * (max_depth x min_samples_leaf) grid into one deep fit per m (BASELINE configs[4]).
 * Host-side renumbering of the BFS prefix; sync. */
dt_status dt_tree_truncate(const dt_tree* tree, int32_t depth, dt_tree** out);

/* dt_predict_eval_depths -- held-out metrics of EVERY truncation depth 0..D of the tree in
 * one pass over (X, y): metrics_host[3*l + {0,1,2}] = (MAPE, R^2, adj-R^2) of
 * dt_tree_truncate(tree, l), l = 0..dt_tree_depth(tree) (<= 32).  Sync. */
dt_status dt_predict_eval_depths(const dt_tree* tree, const float* X_dev, const double* y_dev,
                                 int64_t n, int32_t d, int32_t p, void* stream,
                                 double* metrics_host);

/* dt_importances -- feature importances (Table III; "Gini coefficient"
 * read as the mean decrease in SSE, Reading R3): importances_host[f] = sum over nodes split
 * on f of N*imp - N_L*imp_L - N_R*imp_R, normalised to sum 1 (all zero for a single leaf).
 * importances_host has dt_tree_num_features(tree) entries.  Sync. */
dt_status dt_importances(const dt_tree* tree, double* importances_host, void* stream);

/* ------------------------------------------------------------------ random forest - */

/* Random Forest = bagged CART ("an ensemble of Decision
 * Trees", :231 "the decision is taken based on the average value of all included
 * Decision Trees"; Readings R20, R21).  Tree t (0 <= t < n_trees) is exactly dt_fit's
 * tree of its bootstrap sample: the n rows X[idx_t[i]], y[idx_t[i]], i = 0..n-1 in draw
 * order (duplicates count towards min_samples_leaf), all d features at every split.
 * Draw i of tree t (dt_bootstrap): z = seed + 0x9E3779B97F4A7C15 * ((t << 32) + i + 1),
 * z = (z ^ z >> 30) * 0xBF58476D1CE4E5B9, z = (z ^ z >> 27) * 0x94D049BB133111EB,
 * z ^= z >> 31, idx = z mod n (all mod 2^64).  Prediction: the mean of the trees'
 * predictions, summed in fp64 in tree order, then divided by n_trees.
 * dt_forest_fit: X_dev n x d f32 row-major, y_dev n f64 (as dt_fit); n_trees >= 1.  The
 * table is presorted ONCE; tree t's sorted lists are the presorted lists with every
 * entry repeated by its row's draw count (equal x may then sit in another order than the
 * draw order -- no split falls between equal x, so integer-mode trees are identical).
 * Workspace (stream-ordered, pooled, for the duration of the call): dt_fit's plus
 * ~16 B per (row, feature) for the presorted copy.  Returns when every tree is complete.  The forest owns its trees: dt_forest_tree returns a
 * borrowed pointer valid until dt_forest_free.  Errors as dt_fit. */
typedef struct dt_forest dt_forest;
dt_status dt_forest_fit(const float* X_dev, const double* y_dev, int64_t n, int32_t d,
                        int32_t n_trees, int32_t max_depth, int64_t min_samples_leaf,
                        uint64_t seed, void* stream, dt_forest** out);
int32_t dt_forest_num_trees(const dt_forest* forest);
const dt_tree* dt_forest_tree(const dt_forest* forest, int32_t t);
int64_t dt_forest_split_evals(const dt_forest* forest);  /* sum over the trees */
/* yhat_dev[r] = forest mean for row r of X_dev (n x d f32); async on stream. */
dt_status dt_forest_predict(const dt_forest* forest, const float* X_dev, int64_t n, int32_t d,
                            double* yhat_dev, void* stream);
void dt_forest_free(dt_forest* forest);
/* The bootstrap draws of tree t: idx_dev[i], i < n (u32, device); async on stream. */
dt_status dt_bootstrap(uint64_t seed, int32_t tree, int64_t n, uint32_t* idx_dev, void* stream);

/* ------------------------------------------------------------------ KNN ----------- */

/* dt_knn_predict -- KNN regression (Table II :214;
 * sklearn KNeighborsRegressor defaults: uniform weights, Euclidean; Reading R22):
 * yhat_dev[q] = (sum of y over the k nearest training rows, in (distance, row) order) / k,
 * distance(q, x) = fp64 sum over f in feature order of (q_f - x_f)^2, each term fused
 * (acc = fma(df, df, acc), df = (double)q_f - (double)x_f); equal distances go to the
 * lower training row.  Xtr_dev n_train x d f32, ytr_dev n_train f64, Xq_dev n_query x d
 * f32 (row-major, device); 1 <= k <= min(16, n_train); d in 1..8, 10, 12, 16, 32.
 * Brute force, fp64 CUDA cores (bound: the fp64 pipe).  Async on stream. */
dt_status dt_knn_predict(const float* Xtr_dev, const double* ytr_dev, int64_t n_train, int32_t d,
                         const float* Xq_dev, int64_t n_query, int32_t k, double* yhat_dev,
                         void* stream);

/* ------------------------------------------------------------------ LOO ----------- */

/* dt_loo -- leave-one-out refits (BASELINE configs[0]; the paper's 70/30 split, P:197,
 * has no seed, Reading R11): for every i, fit on the other n-1 rows (original relative
 * order) with (max_depth, min_samples_leaf) and predict row i into yhat_oof_dev[i].
 * Each fold is an independent CART exactly as dt_fit would build it.  2 <= n <= 64 and
 * d <= 32 (one fold per CTA, everything in shared memory); larger inputs -> TOO_LARGE.
 * Async on stream. */
dt_status dt_loo(const float* X_dev, const double* y_dev, int64_t n, int32_t d,
                 int32_t max_depth, int64_t min_samples_leaf, double* yhat_oof_dev,
                 void* stream);

/* ------------------------------------------------------------------ generator ----- */

/* dt_gen_table -- synthetic feature table shaped like Eq. 1: rows
 * [row0, row0 + n) of the seeded (CNN, GPU) table, schema S16 (d = 16) or S32 (d = 32),
 * bit-identical to datagen.cnn_gpu_table (recipe in DESIGN.md, "Input recipe").
 * y_dev may be NULL (features only).  real != 0 -> real-valued target, else integer us.
 * cnn_pool_bits / gpu_pool_bits: pool sizes 2^bits.  unit_us: target unit.  Async. */
dt_status dt_gen_table(uint64_t seed, int64_t row0, int64_t n, int32_t d, int32_t real,
                       int32_t cnn_pool_bits, int32_t gpu_pool_bits, double unit_us,
                       float* X_dev, double* y_dev, void* stream);

/* dt_gen_dse -- DSE candidates (BASELINE configs[3]): candidate r is the cross product
 * entry (cnn = r >> gpu_bits, gpu = r & (2^gpu_bits - 1)), S16 features only,
 * bit-identical to datagen.dse_candidates.  Async. */
dt_status dt_gen_dse(uint64_t seed, int64_t row0, int64_t n, int32_t gpu_bits,
                     float* X_dev, void* stream);

/* ------------------------------------------------------------------ multi-GPU ----- */

/* One process (or host thread) per GPU.  Value-range ROW-sharded exact fit (
 * BASELINE north_star "rows shard naturally across the GPUs ... allreduce / allgather of
 * the per-node, per-feature candidate statistics").  Rank p of P
 * passes only ITS rows: X_local_dev (n_local x d f32 row-major) and y_local_dev (n_local
 * f64) are rows row_offset .. row_offset + n_local - 1 of the n_global-row table, ranks
 * in row order (row_offset of rank p = sum of n_local of ranks < p; n_local may be 0).
 *  - presort: a local sort, exact splitters by bisection on the key (flip(x) << 32 | row)
 *    with a sum-allreduce per round, an all-to-all of 16-byte entries (x, row, y): rank p
 *    then holds global sorted positions [p n / P, (p + 1) n / P) of every feature list;
 *  - per level: allgather of the per-node local bests (reduced in rank order: highest
 *    gain, then lowest feature, then lowest position), OR-allreduce of the n_global-bit
 *    go-left map, allgather of the children's boundary records (count, last x, S') ->
 *    the carries of every child segment.  Entries never move between ranks after the
 *    presort.
 * Every rank returns the same tree: identical to dt_fit's in integer mode except the
 * impurity (summed in another order; within 1e-12 relative), within the parity contract
 * otherwise.  Sync (one host synchronisation per level).
 *   dt_comm_unique_id: 128-byte NCCL id, created by rank 0 and broadcast by the caller
 *     (e.g. torch.distributed); dt_comm_init: NCCL communicator of rank `rank` bound to
 *     CUDA device `device` (made current for the calling thread; INVALID_ARG if out of
 *     range); the caller's dt_fit_sharded / dt_eval_sharded run on that device.
 *     libnccl.so.2 is loaded at run time (DT_ERR_NCCL if absent); a 1-rank communicator
 *     runs the real NCCL collectives.
 *   dt_comm_init_local: `world` communicators for host THREADS of one process (device
 *     copies behind a host barrier), e.g. to run the sharded path on a single GPU.
 * Errors: as dt_fit; INVALID_ARG also for row_offset + n_local > n_global; NCCL. */
typedef struct dt_comm dt_comm;
int32_t dt_comm_unique_id_bytes(void);
dt_status dt_comm_unique_id(void* id_out);
dt_status dt_comm_init(const void* id, int32_t rank, int32_t world, int32_t device, dt_comm** out);
dt_status dt_comm_init_local(int32_t world, dt_comm** comms_out);
void dt_comm_free(dt_comm* comm);
int32_t dt_comm_rank(const dt_comm* comm);
int32_t dt_comm_world(const dt_comm* comm);
dt_status dt_fit_sharded(dt_comm* comm, const float* X_local_dev, const double* y_local_dev, int64_t n_local,
                         int64_t row_offset, int64_t n_global, int32_t d, int32_t max_depth,
                         int64_t min_samples_leaf, void* stream, dt_tree** out);

/* dt_eval_sharded -- MAPE / R^2 / adj-R^2 of rows split over the ranks (SURVEY 8e
 * "Eval"; Table II): each rank reduces its n_local rows (y_dev, yhat_dev f64,
 * device; n_local may be 0) to one partial (sum of |e|/max(|y|, eps), SSE, count and the
 * Welford mean / M2 of y), the partials are allgathered and merged in rank order (Chan),
 * so every rank returns bitwise the same metrics; out->n = the total row count.  Sync. */
dt_status dt_eval_sharded(dt_comm* comm, const double* y_dev, const double* yhat_dev,
                          int64_t n_local, int32_t p, void* stream, dt_metrics* out);

/* ------------------------------------------------------------------ profiling ----- */

/* Measurement hooks used by bench.py (not needed to use the library).  While enabled,
 * every library call records a CUDA event pair on its stream around each kernel it
 * launches, tagged with the kernel kind and the launch's ALGORITHMIC bytes (DESIGN.md,
 * "Roofline"); dt_profile_get synchronises those events and returns, for one kind, the
 * number of launches, the summed device time (ms) and the summed algorithmic bytes.
 * dt_launch_count counts this library's own kernel launches since the last reset.
 * on = 1: events on the stream (a bounded-depth dt_fit then enqueues directly instead of
 * replaying its graph); on = 2: dt_fit keeps its cached CUDA graph, captured once more
 * with event-record nodes around the same kernel groups, and each replay's times are
 * collected when the call returns; on = 0: off. */
void dt_profile_enable(int on);
void dt_profile_reset(void);
int64_t dt_launch_count(void);
int32_t dt_profile_kinds(void);
dt_status dt_profile_get(int32_t kind, const char** name, int64_t* launches, double* ms,
                         double* alg_bytes);

/* ------------------------------------------------------------------ memory -------- */

/* Workspace is kept between calls so that repeated fits allocate nothing: the cached
 * CUDA-graph plans of the last two bounded-depth dt_fit inputs (least recently used
 * replaced; buffers ~34 B per training entry, i.e. ~34 * n * d bytes each, plus per-node
 * tables of ~290 B * min(n / m, 2^max_depth) * d; a plan that does not fit beside the
 * other evicts it) and the freed blocks of the device's default memory pool
 * (stream-ordered workspace of dt_fit_grid, dt_forest_fit, dt_fit_sharded, predict and
 * eval calls; nothing else is cached across calls).  dt_release_workspace
 * synchronises the device, frees the cached plans and trims the pool of the CURRENT
 * device to zero, so that a following large allocation (e.g. the 100M x 32 fit of
 * BASELINE configs[2], ~110 GB) can use the whole HBM.  Always safe to call; the next fit
 * re-plans.  Returns DT_OK, or DT_ERR_CUDA if the device synchronisation fails. */
dt_status dt_release_workspace(void);

/* ------------------------------------------------------------------ misc ---------- */

const char* dt_last_error(void);
/* Library build identification, e.g. "libdt sm_100a". */
const char* dt_version(void);

#ifdef __cplusplus
}
#endif
#endif /* DT_H_ */
