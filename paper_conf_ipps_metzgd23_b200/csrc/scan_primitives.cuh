// Segmented block-scan and decoupled look-back primitives used by the fit kernels.
//
// A "segment" is one (node, feature) run of a level's sorted feature list.  Every scan
// payload carries a head flag; combine(a, b) resets at b's head:
//   combine(a, b) = b.flag ? b : a (+) b,   flag = a.flag | b.flag.
// All block scans have a fixed shape (Kogge-Stone within a warp, then across warps), so
// results are bit-reproducible for a given blockDim.  The look-back folds predecessor
// tiles strictly left to right from the nearest tile that holds a final value, which
// makes the carried prefix identical to the sequential tile-by-tile definition whatever
// the timing (deterministic fp64 prefixes).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace dtl {

// ------------------------------------------------------------------ payloads -------

struct SumP {  // segmented prefix of (y - c)
  uint32_t flag;
  double s;
};
__device__ __forceinline__ SumP combine(const SumP& a, const SumP& b) {
  SumP r;
  r.flag = a.flag | b.flag;
  r.s = b.flag ? b.s : __dadd_rn(a.s, b.s);
  return r;
}
__device__ __forceinline__ SumP shfl_up(const SumP& v, int delta) {
  SumP r;
  r.flag = __shfl_up_sync(0xffffffffu, v.flag, delta);
  r.s = __shfl_up_sync(0xffffffffu, v.s, delta);
  return r;
}

struct CntP {  // segmented count of go-left rows (integers: order-independent)
  uint32_t flag;
  uint32_t c;
};
__device__ __forceinline__ CntP combine(const CntP& a, const CntP& b) {
  CntP r;
  r.flag = a.flag | b.flag;
  r.c = b.flag ? b.c : a.c + b.c;
  return r;
}
__device__ __forceinline__ CntP shfl_up(const CntP& v, int delta) {
  CntP r;
  r.flag = __shfl_up_sync(0xffffffffu, v.flag, delta);
  r.c = __shfl_up_sync(0xffffffffu, v.c, delta);
  return r;
}

struct ArgP {  // segmented argmax of the split gain; ties keep the earlier position
  uint32_t flag;
  uint32_t i;     // within-node position (first i rows go left)
  double gain;    // -1 = no valid candidate
  double sl;      // S'_L at that position
};
__device__ __forceinline__ ArgP combine(const ArgP& a, const ArgP& b) {
  if (b.flag) return b;
  ArgP r = (b.gain > a.gain) ? b : a;
  r.flag = a.flag;
  return r;
}
__device__ __forceinline__ ArgP shfl_up(const ArgP& v, int delta) {
  ArgP r;
  r.flag = __shfl_up_sync(0xffffffffu, v.flag, delta);
  r.i = __shfl_up_sync(0xffffffffu, v.i, delta);
  r.gain = __shfl_up_sync(0xffffffffu, v.gain, delta);
  r.sl = __shfl_up_sync(0xffffffffu, v.sl, delta);
  return r;
}

struct StatP {  // segmented node statistics: sum (y - v)^2, min y, max y, sum (y - c)
  uint32_t flag;
  double sse, ymin, ymax, s1;
};
__device__ __forceinline__ StatP combine(const StatP& a, const StatP& b) {
  if (b.flag) return b;
  StatP r;
  r.flag = a.flag;
  r.sse = __dadd_rn(a.sse, b.sse);
  r.ymin = fmin(a.ymin, b.ymin);
  r.ymax = fmax(a.ymax, b.ymax);
  r.s1 = __dadd_rn(a.s1, b.s1);
  return r;
}
__device__ __forceinline__ StatP shfl_up(const StatP& v, int delta) {
  StatP r;
  r.flag = __shfl_up_sync(0xffffffffu, v.flag, delta);
  r.sse = __shfl_up_sync(0xffffffffu, v.sse, delta);
  r.ymin = __shfl_up_sync(0xffffffffu, v.ymin, delta);
  r.ymax = __shfl_up_sync(0xffffffffu, v.ymax, delta);
  r.s1 = __shfl_up_sync(0xffffffffu, v.s1, delta);
  return r;
}

// ------------------------------------------------------------------ block scan -----

// Exclusive segmented scan over the block (threads in order).  `ident` is returned to
// thread 0 as its exclusive value.  `agg` receives the whole block's inclusive value.
// smem must hold >= 32 T.  Contains __syncthreads(); call from all threads.
template <class T>
__device__ __forceinline__ T block_exclusive_scan(T v, const T& ident, T& agg, T* smem) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int nw = blockDim.x >> 5;
  // inclusive warp scan
  T inc = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    T o = shfl_up(inc, d);
    if (lane >= d) inc = combine(o, inc);
  }
  if (lane == 31) smem[w] = inc;
  __syncthreads();
  if (w == 0) {
    T wv = (lane < nw) ? smem[lane] : ident;
    T wi = wv;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      T o = shfl_up(wi, d);
      if (lane >= d) wi = combine(o, wi);
    }
    // exclusive prefix of warp aggregates, stored at smem[lane]; aggregate at smem[nw]
    T ex = shfl_up(wi, 1);
    if (lane == 0) ex = ident;
    __syncwarp();
    if (lane < nw) smem[lane] = ex;
    if (lane == nw - 1) smem[nw] = wi;
  }
  __syncthreads();
  const T wpre = smem[w];
  agg = smem[nw];
  T ex = shfl_up(inc, 1);
  T res;
  if (lane == 0) res = wpre;
  else res = (w == 0) ? ex : combine(wpre, ex);
  if (w == 0 && lane == 0) res = ident;
  __syncthreads();  // smem reusable afterwards
  return res;
}

// ------------------------------------------------------------------ look-back ------

// Per-tile status word: 0 = nothing, 1 = aggregate published, 2 = inclusive published.
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

template <class T>
struct TileSlots {
  uint32_t* status;  // [ntiles]
  T* agg;            // [ntiles]
  T* inc;            // [ntiles]
};

template <class T>
__device__ __forceinline__ T ldcg(const T* p) {
  // L1-bypassing load of a small POD (values published by other CTAs).
  static_assert(sizeof(T) % 4 == 0, "POD of 32-bit words");
  T r;
  const uint32_t* s = reinterpret_cast<const uint32_t*>(p);
  uint32_t* d = reinterpret_cast<uint32_t*>(&r);
#pragma unroll
  for (int i = 0; i < (int)(sizeof(T) / 4); ++i) d[i] = __ldcg(s + i);
  return r;
}

template <class T>
__device__ __forceinline__ void publish(TileSlots<T> ts, int64_t tile, const T& v, uint32_t state) {
  if (state == 1) ts.agg[tile] = v;
  else ts.inc[tile] = v;
  __threadfence();
  st_release(ts.status + tile, state);
}

// Called by ONE thread.  Returns the exclusive carry for `tile`: the strict left-to-right
// fold of every predecessor tile back to the nearest one holding a final value (status 2,
// or an aggregate that contains a segment head; tile 0's predecessor is the identity).
template <class T>
__device__ T lookback(TileSlots<T> ts, int64_t tile, const T& ident) {
  int64_t t = tile - 1;
  uint32_t st = 0;
  while (t >= 0) {
    do { st = ld_acquire(ts.status + t); } while (st == 0);
    if (st == 2) break;
    if (ldcg(ts.agg + t).flag) break;
    --t;
  }
  T acc = ident;
  if (t >= 0) acc = (st == 2) ? ldcg(ts.inc + t) : ldcg(ts.agg + t);
  for (int64_t u = t + 1; u < tile; ++u) acc = combine(acc, ldcg(ts.agg + u));
  return acc;
}

}  // namespace dtl
