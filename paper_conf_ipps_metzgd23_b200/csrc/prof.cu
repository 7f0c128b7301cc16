// Per-kernel profiling of libdt: CUDA events recorded on the launching stream around
// each kernel (only while enabled), algorithmic bytes per launch, and a launch counter.
// bench.py reads these to report the roofline of the dominant kernel.
// Mode 1: events on the stream (a bounded-depth dt_fit then enqueues directly, no graph).
// Mode 2: dt_fit keeps its CUDA-graph replay; the graph is captured with event-record
// nodes around the same kernel groups, and each replay's times are collected after it.
#include <mutex>
#include <string>
#include <vector>

#include "dt_internal.cuh"

namespace dtl {

namespace {
struct Rec {
  int kind;
  cudaEvent_t a, b;  // null: a collected graph record (ms below)
  double bytes;
  double ms;
};
std::mutex g_mu;
bool g_on = false;
int g_mode = 0;
thread_local std::vector<GRec>* t_cap = nullptr;
constexpr int kGraphTag = 0x40000000;
std::vector<Rec> g_recs;
long long g_launches = 0;
const char* kNames[] = {"presort_keys", "presort_sort", "presort_build", "root_stats",
                        "agg", "select", "number", "goleft", "fused", "predict",
                        "eval", "loo", "gen", "memset"};
constexpr int kNumKinds = sizeof(kNames) / sizeof(kNames[0]);
}  // namespace

int prof_begin(int kind, cudaStream_t s, int nlaunch) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_launches += nlaunch;
  if (!g_on) return -1;
  if (t_cap) {  // capturing a profiled fit graph: event-record nodes
    GRec r{kind, nullptr, nullptr, 0.0};
    cudaEventCreate(&r.a);
    cudaEventCreate(&r.b);
    cudaEventRecordWithFlags(r.a, s, cudaEventRecordExternal);
    t_cap->push_back(r);
    return kGraphTag | (int)(t_cap->size() - 1);
  }
  Rec r;
  r.kind = kind;
  r.bytes = 0.0;
  r.ms = 0.0;
  cudaEventCreate(&r.a);
  cudaEventCreate(&r.b);
  cudaEventRecord(r.a, s);
  g_recs.push_back(r);
  return (int)g_recs.size() - 1;
}

void prof_end(int idx, cudaStream_t s, double bytes) {
  if (idx < 0) return;
  std::lock_guard<std::mutex> lk(g_mu);
  if (idx & kGraphTag) {
    GRec& r = (*t_cap)[(size_t)(idx & ~kGraphTag)];
    r.bytes = bytes;
    cudaEventRecordWithFlags(r.b, s, cudaEventRecordExternal);
    return;
  }
  g_recs[(size_t)idx].bytes = bytes;
  cudaEventRecord(g_recs[(size_t)idx].b, s);
}

void prof_set_bytes(int idx, double bytes) {
  if (idx < 0) return;
  std::lock_guard<std::mutex> lk(g_mu);
  if (idx & kGraphTag) (*t_cap)[(size_t)(idx & ~kGraphTag)].bytes = bytes;
  else g_recs[(size_t)idx].bytes = bytes;
}

bool prof_enabled() {
  std::lock_guard<std::mutex> lk(g_mu);
  return g_on;
}

bool prof_graph_mode() {
  std::lock_guard<std::mutex> lk(g_mu);
  return g_on && g_mode == 2;
}

void prof_capture_target(std::vector<GRec>* v) { t_cap = v; }

void prof_collect_graph(const std::vector<GRec>& v) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g_on) return;
  for (const GRec& r : v) {
    float f = 0.f;
    if (cudaEventElapsedTime(&f, r.a, r.b) != cudaSuccess) continue;
    g_recs.push_back(Rec{r.kind, nullptr, nullptr, r.bytes, (double)f});
  }
}

void prof_destroy_graph_recs(std::vector<GRec>& v) {
  for (GRec& r : v) {
    cudaEventDestroy(r.a);
    cudaEventDestroy(r.b);
  }
  v.clear();
}

void prof_add_launches(long long n) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_launches += n;
}

}  // namespace dtl

using namespace dtl;

extern "C" {

void dt_profile_enable(int on) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_on = on != 0;
  g_mode = on;
}

void dt_profile_reset(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  for (Rec& r : g_recs) {
    if (!r.a) continue;
    cudaEventDestroy(r.a);
    cudaEventDestroy(r.b);
  }
  g_recs.clear();
  g_launches = 0;
}

int64_t dt_launch_count(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  return g_launches;
}

int32_t dt_profile_kinds(void) { return kNumKinds; }

dt_status dt_profile_get(int32_t kind, const char** name, int64_t* launches, double* ms,
                         double* alg_bytes) {
  if (kind < 0 || kind >= kNumKinds) return fail(DT_ERR_INVALID_ARG, "dt_profile_get: bad kind");
  std::lock_guard<std::mutex> lk(g_mu);
  int64_t cnt = 0;
  double t = 0.0, by = 0.0;
  for (Rec& r : g_recs) {
    if (r.kind != kind) continue;
    if (!r.a) {
      t += r.ms;
      by += r.bytes;
      ++cnt;
      continue;
    }
    cudaError_t e = cudaEventSynchronize(r.b);
    if (e != cudaSuccess) return cuda_fail(e, "cudaEventSynchronize", __FILE__, __LINE__);
    float f = 0.f;
    e = cudaEventElapsedTime(&f, r.a, r.b);
    if (e != cudaSuccess) return cuda_fail(e, "cudaEventElapsedTime", __FILE__, __LINE__);
    t += f;
    by += r.bytes;
    ++cnt;
  }
  if (name) *name = kNames[kind];
  if (launches) *launches = cnt;
  if (ms) *ms = t;
  if (alg_bytes) *alg_bytes = by;
  return DT_OK;
}

}  // extern "C"
