// Per-kernel profiling of libdt: CUDA events recorded on the launching stream around
// each kernel (only while enabled), algorithmic bytes per launch, and a launch counter.
// bench.py reads these to report the roofline of the dominant kernel.
#include <mutex>
#include <string>
#include <vector>

#include "dt_internal.cuh"

namespace dtl {

namespace {
struct Rec {
  int kind;
  cudaEvent_t a, b;
  double bytes;
};
std::mutex g_mu;
bool g_on = false;
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
  Rec r;
  r.kind = kind;
  r.bytes = 0.0;
  cudaEventCreate(&r.a);
  cudaEventCreate(&r.b);
  cudaEventRecord(r.a, s);
  g_recs.push_back(r);
  return (int)g_recs.size() - 1;
}

void prof_end(int idx, cudaStream_t s, double bytes) {
  if (idx < 0) return;
  std::lock_guard<std::mutex> lk(g_mu);
  g_recs[(size_t)idx].bytes = bytes;
  cudaEventRecord(g_recs[(size_t)idx].b, s);
}

void prof_set_bytes(int idx, double bytes) {
  if (idx < 0) return;
  std::lock_guard<std::mutex> lk(g_mu);
  g_recs[(size_t)idx].bytes = bytes;
}

bool prof_enabled() {
  std::lock_guard<std::mutex> lk(g_mu);
  return g_on;
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
}

void dt_profile_reset(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  for (Rec& r : g_recs) {
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
