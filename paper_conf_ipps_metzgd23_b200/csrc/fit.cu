// Exact greedy CART regression fit on B200 ("Decision Tree regression";
// split rule, tie rule, threshold and leaf rules: DESIGN.md Readings R1-R10, R19).
//
// Level-synchronous, exact (every feature, every threshold, every node):
//   presort (once)   X row-major -> per-feature lists sorted by (x, row id), SoA
//                    {x f32, row u32, y f64 or int32 (R24)}; batched tile LSD radix sort
//                    of flip(x) with the row id as value (stable: ties keep row order).
//   per level l:     scan      segmented prefix of (y - c_node) over every (node, feature)
//                              segment (three fixed-shape phases: chunk aggregates,
//                              chunk-carry scan, main pass), gain at every
//                              valid position, per-(node,feature) argmax pieces, and
//                              per-node SSE / min / max from the feature-0 list;
//                    select    per node: combine pieces, leaf rules, best feature;
//                    number    BFS numbering of the children, child statistics, offsets;
//                    goleft    bit per row: 1 if the row goes to the left child;
//                    partition stable partition of every feature list into the children
//                              (sorted order preserved, rows of leaves dropped).
// No host synchronisation inside the level loop (counts live on the device); kernels
// are persistent and read the level's node/entry counts from device memory.

#include <math.h>
#include <stdio.h>

#include <algorithm>
#include <memory>
#include <mutex>
#include <vector>

#include "dt_internal.cuh"
#include "bulk.cuh"
#include "scan_primitives.cuh"

namespace dtl {

namespace {

constexpr int kThreads = 256;
#ifndef DT_KITEMS
#define DT_KITEMS 8  // entries per lane of a warp chunk (chunk = 32 x kItems)
#endif
constexpr int kItems = DT_KITEMS;

// Per-level node record (level-local index k).
struct NodeL {
  uint32_t start;  // first position of the node in every feature list of this level
  uint32_t N;      // rows
  int32_t id;      // BFS index in the output node array
  int32_t searchable;
  double c;        // centre (integer mode: floor(S/N); real mode: value)
  double sc;       // S' = sum over the node's rows of (y - c)
  double v;        // value = mean y
  double pad;
};

struct Decision {
  int32_t f;     // split feature (global index), -1 = leaf
  uint32_t nl;   // rows going left (first nl in f-order)
  int32_t floc;  // local list index of f on this rank, -1 if another rank owns f
  int32_t pad;
  double sl;     // S'_L (parent-centred) at the split
  double thr;    // threshold
};

// Per-node result of one rank's local split search (exchanged across ranks).
struct ExchRec {
  double gain;          // -1 = no valid candidate on this rank
  double sl, thr;
  uint32_t i;
  int32_t gf;           // global feature index of the local best
  double sse, ymin, ymax, s1;  // node statistics from this rank's first feature list
};

struct Ctl {
  unsigned long long A[2];  // active entries per feature list, by level parity
  uint32_t K[2];            // nodes at the level, by level parity
  int32_t next_id;          // number of output nodes allocated so far
  int32_t int_mode;
  unsigned long long split_evals;
  int32_t max_depth_seen;
  int32_t nonfinite;
  // root reduction
  double ysum, ymin, ymax, ysc;
  int32_t all_integral;
  int32_t y32;  // the level lists hold y as int32 (Reading R24)
  // chunk lists of the level (single-segment chunks from the front, others from the back)
  uint32_t scnt[2];  // scan: singles, others
  uint32_t pcnt[2];  // partition: singles, others
  uint32_t ticket;   // chunk_scan_kernel: blocks done (the last one computes the block carries)
  uint32_t pad2;
};

struct LevelLog {  // per-level counts, for algorithmic-byte accounting (profiling)
  unsigned long long A, A_next;
  uint32_t K, K_next;
};
constexpr int kMaxLogLevels = 4096;

struct Cand {  // best candidate of one segment piece
  double gain;
  double sl;
  uint32_t i;
  uint32_t kf;     // segment id k*d + f
  uint32_t level;  // level that wrote the record
  uint32_t pad;
};

struct Stat {
  double sse, ymin, ymax, s1;  // s1 = sum (y - c) over the piece
};

// L2 (coherent) loads of a carry payload written by other blocks of the same launch.
__device__ __forceinline__ SumP ld_cg(const SumP* p) {
  SumP r;
  r.flag = __ldcg(&p->flag);
  r.s = __ldcg(&p->s);
  return r;
}
__device__ __forceinline__ CntP ld_cg(const CntP* p) {
  CntP r;
  r.flag = __ldcg(&p->flag);
  r.c = __ldcg(&p->c);
  return r;
}

// Per-level descriptor of the segment holding the FIRST entry of each warp chunk
// (kChunkW entries): one independent load per chunk instead of a dependent lookup chain.
struct __align__(64) ChunkDesc {  // 64 B: one bulk copy
  int64_t start, end;  // global list positions of the segment
  uint32_t k;
  int32_t f;
  double c, sc, v;     // node centre, centred sum, value
  uint32_t N;
  int32_t srch;
};
static_assert(sizeof(ChunkDesc) == 64, "ChunkDesc is copied with one 64-byte bulk copy");
struct PartDesc {
  int64_t start, end;
  uint32_t k;
  int32_t f;
  uint32_t nl, ns;     // decision: rows left, left-child start in the next lists
  int32_t split;
  uint32_t pad;
};

__device__ __forceinline__ uint32_t flip_f32(float x) {
  uint32_t u = __float_as_uint(x);
  if ((u << 1) == 0) u = 0;  // canonicalise -0.0 to +0.0 (equal under f32 compare)
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ __forceinline__ float unflip_f32(uint32_t k) {
  uint32_t u = (k & 0x80000000u) ? (k & 0x7fffffffu) : ~k;
  return __uint_as_float(u);
}

__device__ __forceinline__ long long floor_div_ll(long long a, long long b) {
  long long q = a / b, r = a % b;
  return (r != 0 && r < 0) ? q - 1 : q;
}

// Binary search: largest k in [0, K) with nodes[k].start <= q.
__device__ __forceinline__ uint32_t find_node(const NodeL* __restrict__ nodes, uint32_t K, uint32_t q) {
  uint32_t lo = 0, hi = K;  // invariant: nodes[lo].start <= q < nodes[hi].start
  while (hi - lo > 1) {
    uint32_t mid = (lo + hi) >> 1;
    if (__ldg(&nodes[mid].start) <= q) lo = mid; else hi = mid;
  }
  return lo;
}

// ----------------------------------------------------------------------------- root --

struct RootPart {
  double s, c;  // Neumaier sum
  double mn, mx;
  int integral, finite;
};

__device__ __forceinline__ void neu_add(double& s, double& c, double v) {
  double t = __dadd_rn(s, v);
  if (fabs(s) >= fabs(v)) c = __dadd_rn(c, __dadd_rn(__dsub_rn(s, t), v));
  else c = __dadd_rn(c, __dadd_rn(__dsub_rn(v, t), s));
  s = t;
}

// Deterministic two-level reduction of y: Neumaier sum, min, max, integrality, finiteness.
__global__ void __launch_bounds__(256) root_reduce_kernel(const double* __restrict__ y, int64_t n,
                                                          int64_t chunk, RootPart* parts) {
  const int64_t lo = (int64_t)blockIdx.x * chunk, hi = min(n, lo + chunk);
  RootPart p{0, 0, INFINITY, -INFINITY, 1, 1};
  for (int64_t r = lo + threadIdx.x; r < hi; r += blockDim.x) {
    double v = y[r];
    if (!isfinite(v)) p.finite = 0;
    if (floor(v) != v) p.integral = 0;
    neu_add(p.s, p.c, v);
    p.mn = fmin(p.mn, v);
    p.mx = fmax(p.mx, v);
  }
  __shared__ RootPart sh[256];
  sh[threadIdx.x] = p;
  __syncthreads();
  for (int off = 128; off > 0; off >>= 1) {
    if (threadIdx.x < off) {
      RootPart& a = sh[threadIdx.x];
      const RootPart& b = sh[threadIdx.x + off];
      neu_add(a.s, a.c, b.s);
      neu_add(a.s, a.c, b.c);
      a.mn = fmin(a.mn, b.mn);
      a.mx = fmax(a.mx, b.mx);
      a.integral &= b.integral;
      a.finite &= b.finite;
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) parts[blockIdx.x] = sh[0];
}

__global__ void root_finalize_kernel(const RootPart* parts, int nparts, int64_t n, Ctl* ctl) {
  if (threadIdx.x != 0) return;
  double s = 0, c = 0, mn = INFINITY, mx = -INFINITY;
  int integral = 1, finite = 1;
  for (int i = 0; i < nparts; ++i) {
    neu_add(s, c, parts[i].s);
    neu_add(s, c, parts[i].c);
    mn = fmin(mn, parts[i].mn);
    mx = fmax(mx, parts[i].mx);
    integral &= parts[i].integral;
    finite &= parts[i].finite;
  }
  ctl->ysum = __dadd_rn(s, c);
  ctl->ymin = mn;
  ctl->ymax = mx;
  ctl->all_integral = integral;
  if (!finite) ctl->nonfinite = 1;
  const double amax = fmax(fabs(mn), fabs(mx));
  // Reading R17: integer mode iff every y integral and max|y| * n < 2^52.
  ctl->int_mode = (integral && finite && amax * (double)n < 4503599627370496.0) ? 1 : 0;
  // Reading R24: integral targets with |y| < 2^31 travel through the level lists as int32
  // (4 B instead of 8 per entry; converted exactly to f64 where used)
  ctl->y32 = (ctl->int_mode && amax < 2147483647.0) ? 1 : 0;
}

// S'_0 = sum (y - c0) over all rows (second pass; c0 from the finalised root sum).
__global__ void __launch_bounds__(256) root_center_kernel(const double* __restrict__ y, int64_t n,
                                                          int64_t chunk, const Ctl* ctl, double* parts) {
  const int64_t lo = (int64_t)blockIdx.x * chunk, hi = min(n, lo + chunk);
  double c0;
  if (ctl->int_mode) c0 = (double)floor_div_ll((long long)ctl->ysum, (long long)n);
  else c0 = __ddiv_rn(ctl->ysum, (double)n);
  double s = 0, cc = 0;
  for (int64_t r = lo + threadIdx.x; r < hi; r += blockDim.x) neu_add(s, cc, __dsub_rn(y[r], c0));
  __shared__ double sh[256];
  sh[threadIdx.x] = __dadd_rn(s, cc);
  __syncthreads();
  for (int off = 128; off > 0; off >>= 1) {
    if (threadIdx.x < off) sh[threadIdx.x] = __dadd_rn(sh[threadIdx.x], sh[threadIdx.x + off]);
    __syncthreads();
  }
  if (threadIdx.x == 0) parts[blockIdx.x] = sh[0];
}

__global__ void root_init_kernel(const double* parts, int nparts, int64_t n, int32_t max_depth,
                                 int64_t min_leaf, Ctl* ctl, NodeL* nodes0) {
  if (threadIdx.x != 0) return;
  double s = 0, cc = 0;
  for (int i = 0; i < nparts; ++i) neu_add(s, cc, parts[i]);
  NodeL nd;
  nd.start = 0;
  nd.N = (uint32_t)n;
  nd.id = 0;
  nd.searchable = (max_depth != 0 && n >= 2 * min_leaf) ? 1 : 0;
  if (ctl->int_mode) {
    nd.c = (double)floor_div_ll((long long)ctl->ysum, (long long)n);
    nd.v = __ddiv_rn(ctl->ysum, (double)n);
    nd.sc = ctl->ysum - nd.c * (double)n;  // exact in integer mode
  } else {
    nd.v = __ddiv_rn(ctl->ysum, (double)n);
    nd.c = nd.v;
    nd.sc = __dadd_rn(s, cc);
  }
  nd.pad = 0;
  nodes0[0] = nd;
  ctl->ysc = nd.sc;
  ctl->A[0] = (unsigned long long)n;
  ctl->K[0] = 1;
  ctl->next_id = 1;
  ctl->split_evals = 0;
  ctl->max_depth_seen = 0;
}

// ----------------------------------------------------------------------------- presort --

// keys[f*n + r] = f << 32 | flip(x[r][f]); vals = r.  X row-major -> feature-major via smem.
// Feature sharding: this rank's local feature j is global column j * world + rank of the
// row-major X (row stride dg); keys are built for the d local features only.
__global__ void __launch_bounds__(256) presort_keys_kernel(const float* __restrict__ X, int64_t n, int d,
                                                           uint32_t* __restrict__ keys,
                                                           uint32_t* __restrict__ vals, Ctl* ctl, int dg,
                                                           int world, int rank, int rb) {
  extern __shared__ float tileX[];  // rb rows x dg
  const int64_t r0 = (int64_t)blockIdx.x * rb;
  const int rows = (int)min((int64_t)rb, n - r0);
  const int64_t base = r0 * dg;
  const int tot = rows * dg;
  bool bad = false;
  for (int i = threadIdx.x; i < tot; i += blockDim.x) {
    float v = X[base + i];
    if (!isfinite(v)) bad = true;
    tileX[i] = v;
  }
  if (__syncthreads_or(bad) && threadIdx.x == 0) ctl->nonfinite = 1;
  for (int f = 0; f < d; ++f) {
    if (threadIdx.x < rows) {
      const int64_t r = r0 + threadIdx.x;
      const float v = tileX[threadIdx.x * dg + f * world + rank];
      keys[(int64_t)f * n + r] = flip_f32(v);
      vals[(int64_t)f * n + r] = (uint32_t)r;
    }
  }
}

// SoA level-0 lists from the sorted pairs: x = unflip(key), row = val, y = y[row].
__global__ void __launch_bounds__(256) presort_build_kernel(const uint32_t* __restrict__ keys,
                                                            const uint32_t* __restrict__ vals,
                                                            const double* __restrict__ y, int64_t total,
                                                            float* __restrict__ lx, uint32_t* __restrict__ lr,
                                                            double* __restrict__ ly, const Ctl* ctl) {
  const bool y32 = ctl->y32 != 0;
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < total;
       p += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t r = vals[p];
    lx[p] = unflip_f32(keys[p]);
    lr[p] = r;
    const double v = __ldg(y + r);
    if (y32) reinterpret_cast<int32_t*>(ly)[p] = (int32_t)v;
    else ly[p] = v;
  }
}

// Batched LSD radix sort of the d per-feature key lists (any n < 2^32): 4 passes
// of 8-bit digits; per pass three launches, each over all d features (grid.y = feature):
//   rs_count:   per-tile digit counts;
//   rs_offset:  per (feature, digit) exclusive scan of the counts over the tiles, and the
//               digit totals;
//   rs_scatter: every key's stable rank inside its tile (warp match_any per step of 32
//               keys + per-warp digit counters; keys in tile order), then its destination
//               = (keys of smaller digits) + (same digit, earlier tiles) + rank.
// Stable within a feature, so equal keys keep the row order: (x, row id) order (R6).
constexpr int kTS = 256, kTI = 8, kTile = kTS * kTI;

__global__ void __launch_bounds__(kTS) rs_count_kernel(const uint32_t* __restrict__ keys, int64_t n, int shift,
                                                       int tiles, uint32_t* __restrict__ cnt) {
  __shared__ uint32_t h[256];
  const int f = blockIdx.y, tile = blockIdx.x;
  h[threadIdx.x] = 0u;
  __syncthreads();
  const int64_t base = (int64_t)f * n + (int64_t)tile * kTile;
  const int m = (int)min((int64_t)kTile, n - (int64_t)tile * kTile);
  for (int i = threadIdx.x; i < m; i += kTS) atomicAdd(&h[(__ldg(keys + base + i) >> shift) & 255u], 1u);
  __syncthreads();
  cnt[((int64_t)f * 256 + threadIdx.x) * tiles + tile] = h[threadIdx.x];
}

// grid (256 digits, d features): exclusive prefix of one digit's counts over the tiles
// (fixed shape; integers), and the digit's total.
__global__ void __launch_bounds__(1024) rs_offset_kernel(const uint32_t* __restrict__ cnt, int tiles,
                                                         uint32_t* __restrict__ off, uint32_t* __restrict__ tot) {
  __shared__ uint32_t sw[32];
  __shared__ uint32_t s_run;
  const int64_t base = ((int64_t)blockIdx.y * 256 + blockIdx.x) * tiles;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (threadIdx.x == 0) s_run = 0u;
  __syncthreads();
  for (int t0 = 0; t0 < tiles; t0 += blockDim.x) {
    const int t = t0 + threadIdx.x;
    const uint32_t c = (t < tiles) ? __ldg(cnt + base + t) : 0u;
    uint32_t inc = c;
#pragma unroll
    for (int dd = 1; dd < 32; dd <<= 1) {
      const uint32_t o = __shfl_up_sync(0xffffffffu, inc, dd);
      if (lane >= dd) inc += o;
    }
    if (lane == 31) sw[w] = inc;
    __syncthreads();
    if (w == 0) {
      const uint32_t v = (lane < (int)(blockDim.x >> 5)) ? sw[lane] : 0u;
      uint32_t vi = v;
#pragma unroll
      for (int dd = 1; dd < 32; dd <<= 1) {
        const uint32_t o = __shfl_up_sync(0xffffffffu, vi, dd);
        if (lane >= dd) vi += o;
      }
      sw[lane] = vi - v;  // exclusive prefix of the warp totals
    }
    __syncthreads();
    const uint32_t run = s_run;
    if (t < tiles) off[base + t] = run + sw[w] + inc - c;
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) s_run = run + sw[w] + inc;
    __syncthreads();
  }
  if (threadIdx.x == 0) tot[(int64_t)blockIdx.y * 256 + blockIdx.x] = s_run;
}

#ifndef DT_RS_MINB
#define DT_RS_MINB 4  // 4 CTAs/SM (64 registers): more tiles in flight (measured 4.04 -> 3.95 ms/step)
#endif
__global__ void __launch_bounds__(kTS, DT_RS_MINB) rs_scatter_kernel(const uint32_t* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                         uint32_t* __restrict__ kout, uint32_t* __restrict__ vout,
                                                         int64_t n, int shift, int tiles, const uint32_t* __restrict__ off,
                                                         const uint32_t* __restrict__ tot) {
  __shared__ uint32_t wc[kTS / 32][256];  // per-warp digit counters -> per-warp prefixes
  __shared__ uint32_t s_base[256];        // digit base of this tile: smaller digits + earlier tiles
  __shared__ uint32_t s_start[256];       // digit starts inside the tile
  __shared__ uint32_t skey[kTile], sval[kTile];
  __shared__ uint32_t sw[kTS / 32], sw2[kTS / 32];
  const int f = blockIdx.y, tile = blockIdx.x;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t base = (int64_t)f * n + (int64_t)tile * kTile;
  const int m = (int)min((int64_t)kTile, n - (int64_t)tile * kTile);
  for (int q = lane; q < 256; q += 32) wc[w][q] = 0u;
  // keys of warp w: tile positions w * 256 + j * 32 + lane (coalesced, in tile order)
  uint32_t keys[kTI], vals[kTI], rk[kTI];
#pragma unroll
  for (int j = 0; j < kTI; ++j) {
    const int i = w * 256 + j * 32 + lane;
    keys[j] = (i < m) ? __ldg(kin + base + i) : 0u;
    vals[j] = (i < m) ? __ldg(vin + base + i) : 0u;
  }
  __syncwarp();
  const uint32_t lt = (1u << lane) - 1u;
#pragma unroll
  for (int j = 0; j < kTI; ++j) {
    const int i = w * 256 + j * 32 + lane;
    const bool v = i < m;
    const uint32_t dg = v ? ((keys[j] >> shift) & 255u) : 256u;  // padding: its own class
    const uint32_t peers = __match_any_sync(0xffffffffu, dg);
    const uint32_t before = wc[w][dg & 255u];
    rk[j] = before + __popc(peers & lt);
    __syncwarp();
    if (v && (peers & lt) == 0u) wc[w][dg] = before + __popc(peers);  // lowest peer updates
    __syncwarp();
  }
  __syncthreads();
  // thread = digit: exclusive prefix over the warps, the tile's digit starts (exclusive
  // scan of its digit counts) and the digit's global base for this tile
  {
    const int dgt = threadIdx.x;
    uint32_t run = 0u;
#pragma unroll
    for (int q = 0; q < kTS / 32; ++q) {
      const uint32_t c = wc[q][dgt];
      wc[q][dgt] = run;
      run += c;
    }
    uint32_t inc = run;  // tile count of this digit
#pragma unroll
    for (int dd = 1; dd < 32; dd <<= 1) {
      const uint32_t o = __shfl_up_sync(0xffffffffu, inc, dd);
      if (lane >= dd) inc += o;
    }
    if (lane == 31) sw[w] = inc;
    // exclusive prefix of the digit totals of this feature
    const uint32_t t = __ldg(tot + (int64_t)f * 256 + dgt);
    uint32_t tinc = t;
#pragma unroll
    for (int dd = 1; dd < 32; dd <<= 1) {
      const uint32_t o = __shfl_up_sync(0xffffffffu, tinc, dd);
      if (lane >= dd) tinc += o;
    }
    if (lane == 31) sw2[w] = tinc;
    __syncthreads();
    uint32_t wp = 0u, wp2 = 0u;
    for (int q = 0; q < w; ++q) { wp += sw[q]; wp2 += sw2[q]; }
    s_start[dgt] = wp + inc - run;
    s_base[dgt] = wp2 + tinc - t + __ldg(off + ((int64_t)f * 256 + dgt) * tiles + tile);
  }
  __syncthreads();
  // local (tile-sorted) order in shared memory, then coalesced runs to global memory
#pragma unroll
  for (int j = 0; j < kTI; ++j) {
    const int i = w * 256 + j * 32 + lane;
    if (i < m) {
      const uint32_t dg = (keys[j] >> shift) & 255u;
      const uint32_t lp = s_start[dg] + wc[w][dg] + rk[j];
      skey[lp] = keys[j];
      sval[lp] = vals[j];
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < m; i += kTS) {
    const uint32_t key = skey[i];
    const uint32_t dg = (key >> shift) & 255u;
    const int64_t dst = (int64_t)f * n + s_base[dg] + ((uint32_t)i - s_start[dg]);
    kout[dst] = key;
    vout[dst] = sval[i];
  }
}

// ----------------------------------------------------------------------------- scan ----

// Appends chunk c to a level's chunk list: single-segment chunks from the front, the
// others from the back (warp-aggregated atomics; the order inside a list is irrelevant,
// every chunk's results are independent of when it is processed).
__device__ __forceinline__ void list_chunk(uint32_t* cnt, uint32_t* list, int64_t nch, int64_t c, bool single) {
  const unsigned am = __activemask();
  const int lane = threadIdx.x & 31;
  const unsigned ms = __ballot_sync(am, single);
  const int leader = __ffs(am) - 1;
  uint32_t bs = 0, bg = 0;
  if (lane == leader) {
    bs = atomicAdd(cnt, (uint32_t)__popc(ms));
    bg = atomicAdd(cnt + 1, (uint32_t)__popc(am & ~ms));
  }
  bs = __shfl_sync(am, bs, leader);
  bg = __shfl_sync(am, bg, leader);
  const unsigned lt = (1u << lane) - 1u;
  if (single) list[bs + __popc(ms & lt)] = (uint32_t)c;
  else list[nch - 1 - (bg + __popc(am & ~ms & lt))] = (uint32_t)c;
}

__global__ void __launch_bounds__(256) scan_desc_kernel(const NodeL* __restrict__ nodes, Ctl* ctl,
                                                        int parity, int dl, int chunkw, ChunkDesc* __restrict__ desc,
                                                        uint32_t* __restrict__ list) {
  const uint32_t K = ctl->K[parity];
  const uint64_t A = ctl->A[parity];
  if (blockIdx.x == 0 && threadIdx.x == 0) ctl->pcnt[0] = ctl->pcnt[1] = 0;  // this level's partition lists
  if (K == 0 || A == 0) return;
  const int64_t total = (int64_t)A * dl;
  const int64_t nch = (total + chunkw - 1) / chunkw;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < nch; c += (int64_t)gridDim.x * blockDim.x) {
    const int64_t p = c * chunkw;
    const int f = (int)(p / (int64_t)A);
    const int64_t fbase = (int64_t)f * (int64_t)A;
    const uint32_t k = find_node(nodes, K, (uint32_t)(p - fbase));
    const NodeL nd = nodes[k];
    ChunkDesc d;
    d.start = fbase + nd.start;
    d.end = d.start + nd.N;
    d.k = k;
    d.f = f;
    d.c = nd.c;
    d.sc = nd.sc;
    d.v = nd.v;
    d.N = nd.N;
    d.srch = nd.searchable;
    desc[c] = d;
    list_chunk(ctl->scnt, list, nch, c, d.start <= p && d.end >= p + chunkw);
  }
}

// Cursor over the segments of a level's concatenated feature lists: segment (f, k)
// occupies global positions [f*A + start_k, f*A + start_k + N_k).
struct Seg {
  int64_t start, end, fbase;
  uint32_t k;
  int f;
};
__device__ __forceinline__ void seg_next(Seg& s, const NodeL* __restrict__ nodes, uint32_t K,
                                         uint64_t A) {
  if (++s.k == K) {
    s.k = 0;
    ++s.f;
    s.fbase += (int64_t)A;
  }
  s.start = s.fbase + __ldg(&nodes[s.k].start);
  s.end = s.start + __ldg(&nodes[s.k].N);
}

// Cursor for position p starting from a chunk descriptor's segment (walks forward).
__device__ __forceinline__ void seg_from(Seg& s, int64_t start, int64_t end, uint32_t k, int f,
                                         uint64_t A, int64_t p, const NodeL* __restrict__ nodes,
                                         uint32_t K) {
  s.start = start;
  s.end = end;
  s.k = k;
  s.f = f;
  s.fbase = (int64_t)f * (int64_t)A;
  while (p >= s.end) seg_next(s, nodes, K, A);
}

struct ScanArgs {
  const float* lx;
  const double* ly;
  const NodeL* nodes;
  const Ctl* ctl;
  int parity;
  int dl;          // feature lists present at this level (d, or 1 at the last level)
  int d;           // feature count (slot stride)
  int64_t min_leaf;
  const ChunkDesc* desc;  // per warp chunk
  const uint32_t* list;   // chunk list (scan_desc_kernel): singles first, others from the back
  SumP* chunk_agg;    // [nchunks] phase A: per-warp-chunk aggregate
  SumP* chunk_excl;   // [nchunks] phase B1: exclusive within its block of chunks
  SumP* block_agg;    // [nblocks] phase B1: block aggregates
  SumP* block_carry;  // [nblocks] phase B2: exclusive carry per block of chunks
  Cand* head_cand;  // [K*d]
  Cand* cont_cand;  // [nchunks]
  unsigned long long* slot_gain;  // [K*d] running max gain bits (zero between levels)
  uint32_t level;
  Stat* head_stat;  // [K]
  Stat* cont_stat;  // [nchunks]
};

// Piece record + running per-segment max of the gain (u64 order == f64 order for gains
// >= 0).  The position of the winner is resolved by piece_pos_kernel (lowest position
// among pieces whose gain equals the max), so the result is exact and deterministic.
__device__ __forceinline__ void write_cand(Cand* p, const ArgP& a, uint32_t kf, uint32_t level,
                                           unsigned long long* slot_gain) {
  Cand c;
  c.gain = a.gain;
  c.sl = a.sl;
  c.i = a.i;
  c.kf = kf;
  c.level = level;
  c.pad = 0;
  *p = c;
  if (a.gain >= 0.0) atomicMax(slot_gain + kf, (unsigned long long)__double_as_longlong(a.gain));
}
__device__ __forceinline__ void write_stat(Stat* p, const StatP& a) {
  Stat s;
  s.sse = a.sse;
  s.ymin = a.ymin;
  s.ymax = a.ymax;
  s.s1 = a.s1;
  *p = s;
}

// Gain of candidate "first i rows left" (Reading R19), no FMA contraction:
//   D = S'_L n_R - S'_R n_L,  gain = D^2 / ((N n_L) n_R).
// nl, Nd: the left count and the node size as doubles (exact integers).  Callers in the
// per-item loops pass nl = (double)i0 + j (exact), so no int->f64 conversion (an XU-pipe
// op, the scan's former bottleneck) runs per item; the values are identical.
__device__ __forceinline__ double split_gain_d(double sl, double sc, double nl, double Nd) {
  const double nr = __dsub_rn(Nd, nl);
  const double sr = __dsub_rn(sc, sl);
  const double D = __dsub_rn(__dmul_rn(sl, nr), __dmul_rn(sr, nl));
  return __ddiv_rn(__dmul_rn(D, D), __dmul_rn(__dmul_rn(Nd, nl), nr));
}
__device__ __forceinline__ double split_gain(double sl, double sc, uint32_t i, uint32_t N) {
  return split_gain_d(sl, sc, (double)i, (double)N);
}

// Same D and denominator as split_gain; the quotient via a Newton-refined reciprocal
// (relative error ~3e-16).  Used only to locate the exact argmax (see scan_kernel).
__device__ __forceinline__ double rcp_nr(double x) {
  double r;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
  double e = __fma_rn(-x, r, 1.0);
  r = __fma_rn(r, e, r);
  e = __fma_rn(-x, r, 1.0);
  return __fma_rn(r, e, r);
}
__device__ __forceinline__ double split_gain_approx_d(double sl, double sc, double nl, double Nd) {
  const double nr = __dsub_rn(Nd, nl);
  const double sr = __dsub_rn(sc, sl);
  const double D = __dsub_rn(__dmul_rn(sl, nr), __dmul_rn(sr, nl));
  return __dmul_rn(__dmul_rn(D, D), rcp_nr(__dmul_rn(__dmul_rn(Nd, nl), nr)));
}

// Loads kItems consecutive x (f32) and y (f64) entries starting at p0 (vectorised when
// the whole run is in bounds; p0 is a multiple of kItems, so 16-byte aligned).
// y list element p: int32 storage when y32 (Reading R24), else f64.
__device__ __forceinline__ double yget(const double* __restrict__ ly, int64_t p, bool y32) {
  return y32 ? (double)reinterpret_cast<const int32_t*>(ly)[p] : ly[p];
}

// kItems consecutive y entries from p0 (p0 + kItems <= total; p0 a multiple of kItems).
__device__ __forceinline__ void load_y_vec(const double* __restrict__ ly, int64_t p0, bool y32, double* yv) {
  if (y32) {
    const int4* y4 = reinterpret_cast<const int4*>(reinterpret_cast<const int32_t*>(ly) + p0);
#pragma unroll
    for (int j = 0; j < kItems / 4; ++j) {
      const int4 t = __ldcs(y4 + j);
      yv[4 * j] = (double)t.x; yv[4 * j + 1] = (double)t.y; yv[4 * j + 2] = (double)t.z; yv[4 * j + 3] = (double)t.w;
    }
  } else {
    const double2* y2 = reinterpret_cast<const double2*>(ly + p0);
#pragma unroll
    for (int j = 0; j < kItems / 2; ++j) {
      const double2 t = __ldcs(y2 + j);
      yv[2 * j] = t.x; yv[2 * j + 1] = t.y;
    }
  }
}

// Loads kItems consecutive x (f32) and y entries starting at p0 (vectorised when the
// whole run is in bounds; p0 is a multiple of kItems, so 16-byte aligned).
__device__ __forceinline__ void load_items(const float* __restrict__ lx, const double* __restrict__ ly,
                                           int64_t p0, int64_t total, float* xv, double* yv, bool y32) {
  if (p0 + kItems <= total) {
    const float4* x4 = reinterpret_cast<const float4*>(lx + p0);
#pragma unroll
    for (int j = 0; j < kItems / 4; ++j) {
      const float4 t = __ldcs(x4 + j);
      xv[4 * j] = t.x; xv[4 * j + 1] = t.y; xv[4 * j + 2] = t.z; xv[4 * j + 3] = t.w;
    }
    load_y_vec(ly, p0, y32, yv);
  } else {
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
      const bool ok = p0 + j < total;
      xv[j] = ok ? lx[p0 + j] : 0.f;
      yv[j] = ok ? yget(ly, p0 + j, y32) : 0.0;
    }
  }
}

// Thread aggregate of the segmented sum of (y - c) over my kItems entries (pass 1).
// Shared by the tile-aggregate kernel and the main scan, so both see identical values.
__device__ __forceinline__ SumP thread_sum_agg(const ScanArgs& a, uint32_t K, uint64_t A, int64_t p0,
                                               int64_t total, bool any, bool warp_fast, bool head0,
                                               const Seg& sg, const double* yv, double c_first) {
  SumP tagg{0u, 0.0};
  if (!any) return tagg;
  if (warp_fast) {
    const double c = c_first;
    double t = head0 ? __dsub_rn(yv[0], c) : __dadd_rn(0.0, __dsub_rn(yv[0], c));
#pragma unroll
    for (int j = 1; j < kItems; ++j) t = __dadd_rn(t, __dsub_rn(yv[j], c));
    tagg.flag = head0 ? 1u : 0u;
    tagg.s = t;
  } else {
    Seg s = sg;
    double c = c_first;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
      const int64_t p = p0 + j;
      if (p < total) {
        if (p == s.end) {
          seg_next(s, a.nodes, K, A);
          c = __ldg(&a.nodes[s.k].c);
        }
        const double e = __dsub_rn(yv[j], c);
        if (p == s.start) { tagg.flag = 1u; tagg.s = e; }
        else tagg.s = __dadd_rn(tagg.s, e);
      }
    }
  }
  return tagg;
}

__device__ __forceinline__ void load_y(const double* __restrict__ ly, int64_t p0, int64_t total, double* yv,
                                       bool y32) {
  if (p0 + kItems <= total) {
    load_y_vec(ly, p0, y32, yv);
  } else {
#pragma unroll
    for (int j = 0; j < kItems; ++j) yv[j] = (p0 + j < total) ? yget(ly, p0 + j, y32) : 0.0;
  }
}

// The scan works on WARP CHUNKS of kChunkW = 32 x kItems list entries (lane L owns
// entries [kItems*L, kItems*L + kItems) of its warp's chunk).  All scans inside a chunk
// are warp-shuffle scans (no block barrier); chunk carries come from phase B.
constexpr int kChunkW = 32 * kItems;           // 256 entries
#ifndef DT_BLOCK_CHUNKS
#define DT_BLOCK_CHUNKS 1024  // one chunk per thread (measured: 2048 -> 1024 saves ~1% of the step)
#endif
constexpr int kBlockChunks = DT_BLOCK_CHUNKS;  // chunks per phase-B block (1024 threads)

// Phase A: per-chunk segmented aggregate of (y - c) (reads y only).
// One chunk's segmented aggregate of (y - c) into chunk_agg[ch].
__device__ __forceinline__ void agg_chunk(const ScanArgs& a, uint32_t K, uint64_t A, int64_t total, int64_t ch,
                                          const double* yv, const ChunkDesc& dsc) {
  const int lane = threadIdx.x & 31;
  const int64_t p0 = ch * kChunkW + lane * kItems;
  const bool any = p0 < total;
  if (dsc.start <= ch * kChunkW && dsc.end >= ch * kChunkW + kChunkW) {
    // whole chunk in one segment: the general path's sums without the segment logic
    const bool head = dsc.start == ch * kChunkW;
    const double c = dsc.c;
    double t = (head && lane == 0) ? __dsub_rn(yv[0], c) : __dadd_rn(0.0, __dsub_rn(yv[0], c));
#pragma unroll
    for (int j = 1; j < kItems; ++j) t = __dadd_rn(t, __dsub_rn(yv[j], c));
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const double o = __shfl_up_sync(0xffffffffu, t, d);
      if (lane >= d) t = __dadd_rn(o, t);
    }
    if (lane == 31) a.chunk_agg[ch] = SumP{head ? 1u : 0u, t};
    return;
  }
  Seg sg{0, 0, 0, 0u, 0};
  if (any) seg_from(sg, dsc.start, dsc.end, dsc.k, dsc.f, A, p0, a.nodes, K);
  const bool one_seg = any && (p0 + kItems <= total) && (sg.end >= p0 + kItems);
  const bool warp_fast = __all_sync(0xffffffffu, one_seg || !any);
  const bool head0 = any && (p0 == sg.start);
  const double c_in = (sg.k == dsc.k && sg.f == dsc.f) ? dsc.c : __ldg(&a.nodes[sg.k].c);
  const SumP tagg = thread_sum_agg(a, K, A, p0, total, any, warp_fast, head0, sg, yv, c_in);
  SumP wagg;
  (void)warp_exclusive_scan(tagg, SumP{0u, 0.0}, wagg);
  if (lane == 0) a.chunk_agg[ch] = wagg;
}

// Phase A over the level's full chunks with a per-warp TMA pipeline (kAggStages chunks of
// y and their descriptors in flight per warp: the pass is a pure stream of y); a partial
// last chunk goes through registers.
#ifndef DT_AGG_STAGES
#define DT_AGG_STAGES 3
#endif
constexpr int kAggStages = DT_AGG_STAGES;
struct __align__(128) AggStage {
  double y[kChunkW];  // 256 f64 or 256 int32 (first half)
  ChunkDesc d;
};
constexpr size_t kScanAggSmem = (sizeof(AggStage) + sizeof(uint64_t)) * kAggStages * (kThreads / 32);

__global__ void __launch_bounds__(kThreads) scan_agg_kernel(ScanArgs a) {
  extern __shared__ __align__(128) unsigned char agg_smem[];
  const uint32_t K = a.ctl->K[a.parity];
  const uint64_t A = a.ctl->A[a.parity];
  if (K == 0 || A == 0) return;
  const int64_t total = (int64_t)A * a.dl;
  const int64_t nfull = total / kChunkW;
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const bool y32 = a.ctl->y32 != 0;
  if (gw == 0 && nfull * kChunkW < total) {  // the partial last chunk
    double yv[kItems];
    const int64_t p0 = nfull * kChunkW + lane * kItems;
#pragma unroll
    for (int j = 0; j < kItems; ++j) yv[j] = 0.0;
    if (p0 < total) load_y(a.ly, p0, total, yv, y32);
    agg_chunk(a, K, A, total, nfull, yv, a.desc[nfull]);
  }
  if (gw >= nfull) return;  // warp-uniform
  AggStage* st = reinterpret_cast<AggStage*>(agg_smem) + wib * kAggStages;
  uint64_t* bar = reinterpret_cast<uint64_t*>(agg_smem + sizeof(AggStage) * kAggStages * (kThreads / 32)) +
                  wib * kAggStages;
  const uint32_t ybytes = (uint32_t)(y32 ? sizeof(int32_t) : sizeof(double)) * kChunkW;
  auto issue = [&](int q, int64_t ch) {  // lane 0
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(bar + q, ybytes + (uint32_t)sizeof(ChunkDesc));
    bulk_g2s(st[q].y, reinterpret_cast<const char*>(a.ly) + ch * (int64_t)ybytes, ybytes, bar + q);
    bulk_g2s(&st[q].d, a.desc + ch, sizeof(ChunkDesc), bar + q);
  };
  if (lane == 0) {
    for (int q = 0; q < kAggStages; ++q) mbar_init(bar + q, 1);
    mbar_init_fence();
    for (int q = 0; q < kAggStages; ++q)
      if (gw + q * nw < nfull) issue(q, gw + q * nw);
  }
  __syncwarp();
  int q = 0;
  uint32_t phase = 0;
  for (int64_t ch = gw; ch < nfull; ch += nw) {
    mbar_wait(bar + q, phase);
    double yv[kItems];
    if (y32) {
      const int4* y4 = reinterpret_cast<const int4*>(reinterpret_cast<const int32_t*>(st[q].y) + lane * kItems);
#pragma unroll
      for (int j = 0; j < kItems / 4; ++j) {
        const int4 v = y4[j];
        yv[4 * j] = (double)v.x; yv[4 * j + 1] = (double)v.y; yv[4 * j + 2] = (double)v.z; yv[4 * j + 3] = (double)v.w;
      }
    } else {
      const double2* y2 = reinterpret_cast<const double2*>(st[q].y + lane * kItems);
#pragma unroll
      for (int j = 0; j < kItems / 2; ++j) {
        const double2 v = y2[j];
        yv[2 * j] = v.x; yv[2 * j + 1] = v.y;
      }
    }
    const ChunkDesc dsc = st[q].d;
    __syncwarp();  // every lane has read the stage
    const int64_t nxt = ch + kAggStages * nw;
    if (lane == 0 && nxt < nfull) issue(q, nxt);
    agg_chunk(a, K, A, total, ch, yv, dsc);
    if (++q == kAggStages) { q = 0; phase ^= 1u; }
  }
}

// Phase B: exclusive segmented scan of per-chunk aggregates inside blocks of
// kBlockChunks chunks (kPer per thread sequentially, then a block scan), then -- by the
// last block to finish (ticket) -- the exclusive scan of the block aggregates (carries).
// Fixed shape, so deterministic.  Used for the scan (SumP) and the partition (CntP).
template <class T>
__global__ void __launch_bounds__(1024) chunk_scan_kernel(Ctl* ctl, int parity, int dl,
                                                          const T* __restrict__ chunk_agg,
                                                          T* __restrict__ chunk_excl, T* block_agg,
                                                          T* __restrict__ block_carry) {
  __shared__ T sh[33];
  __shared__ T sh_run;
  __shared__ bool s_last;
  const uint32_t K = ctl->K[parity];
  const uint64_t A = ctl->A[parity];
  const int64_t total = (K == 0) ? 0 : (int64_t)A * dl;
  const int64_t nch = (total + kChunkW - 1) / kChunkW;
  const int64_t b0 = (int64_t)blockIdx.x * kBlockChunks;
  T zero;
  zero.flag = 0u;
  from_bits(zero, 0ull);
  if (b0 < nch) {  // block-uniform
    constexpr int kPer = kBlockChunks / 1024;
    const int64_t c0 = b0 + (int64_t)threadIdx.x * kPer;
    T v[kPer];
    T agg = zero;
#pragma unroll
    for (int q = 0; q < kPer; ++q) {
      v[q] = (c0 + q < nch) ? chunk_agg[c0 + q] : zero;
      agg = (q == 0) ? v[0] : combine(agg, v[q]);
    }
    T bagg;
    T cur = block_exclusive_scan(agg, zero, bagg, sh);
#pragma unroll
    for (int q = 0; q < kPer; ++q) {
      if (c0 + q < nch) chunk_excl[c0 + q] = cur;
      cur = combine(cur, v[q]);
    }
    if (threadIdx.x == 0) block_agg[blockIdx.x] = bagg;
  }
  // the last block to arrive scans the block aggregates
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) s_last = atomicAdd(&ctl->ticket, 1u) == gridDim.x - 1;
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  if (threadIdx.x == 0) {
    ctl->ticket = 0u;  // ready for the next launch
    sh_run = zero;
  }
  const int64_t nb = (nch + kBlockChunks - 1) / kBlockChunks;
  __syncthreads();
  for (int64_t base = 0; base < nb; base += blockDim.x) {
    const int64_t bi = base + threadIdx.x;
    T v = zero;
    if (bi < nb) v = ld_cg(block_agg + bi);
    T chunk;
    const T ex = block_exclusive_scan(v, zero, chunk, sh);
    const T run = sh_run;
    if (bi < nb) block_carry[bi] = combine(run, ex);
    __syncthreads();
    if (threadIdx.x == 0) sh_run = combine(run, chunk);
    __syncthreads();
  }
}

// Whole warp chunk inside ONE segment (a head can only sit at the chunk's first entry) --
// true for nearly every chunk at shallow levels.  Same sums in the same order as the
// general path (thread sums item by item, Kogge-Stone prefix, carry), so the results are
// bitwise identical; the per-chunk argmax is a warp max-reduction + lowest winning lane
// (exact selection, ties to the lowest position like ArgP's combine).
// Valid split positions of one chunk, compacted (position order) for the exact gains.
constexpr int kCompactMax = kChunkW;
struct CompactBuf {
  double sl[kCompactMax];
  uint32_t i[kCompactMax];
};

__device__ __forceinline__ void scan_single(const ScanArgs& a, int64_t ch, int64_t cbase, const ChunkDesc& dsc,
                                            const float* xv, const double* yv, uint32_t m, const SumP& carry,
                                            float xp0, CompactBuf& cb) {
  const int lane = threadIdx.x & 31;
  const bool head = dsc.start == cbase;
  const bool head0 = head && lane == 0;
  const double c = dsc.c;
  double t = head0 ? __dsub_rn(yv[0], c) : __dadd_rn(0.0, __dsub_rn(yv[0], c));
#pragma unroll
  for (int j = 1; j < kItems; ++j) t = __dadd_rn(t, __dsub_rn(yv[j], c));
  double inc = t;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const double o = __shfl_up_sync(0xffffffffu, inc, d);
    if (lane >= d) inc = __dadd_rn(o, inc);
  }
  double S = __shfl_up_sync(0xffffffffu, inc, 1);
  if (lane == 0) S = 0.0;
  if (!head) S = __dadd_rn(carry.s, S);

  // Valid positions (x_prev < x, both children >= m) are few on tied data (a column with
  // V distinct values has < V boundaries per node): the (prefix, position) pairs of the
  // chunk's valid positions are compacted, in position order, into shared memory and the
  // EXACT gain of each is computed once, lane q taking entries q, q + 32, .. (strict >
  // per lane, then a warp (max gain, lowest index) reduction == the lowest position
  // among the maxima).  On tied data one round of 32 gains covers a whole chunk.
  ArgP best{0u, 0xffffffffu, -1.0, 0.0};
  if (dsc.srch) {
    const double sc = dsc.sc;
    const uint32_t N = dsc.N;
    const uint32_t i0 = (uint32_t)(cbase + lane * kItems - dsc.start);
    const uint32_t ilo = m > 1u ? m : 1u, ihi = N - m;
    float xprev = __shfl_up_sync(0xffffffffu, xv[kItems - 1], 1);
    if (lane == 0) xprev = head ? 0.f : xp0;
    uint32_t vm = 0u;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
      const uint32_t i = i0 + j;
      const float xp = (j == 0) ? xprev : xv[j - 1];
      if (i >= ilo && i <= ihi && xp < xv[j]) vm |= 1u << j;
    }
    const uint32_t nv = __popc(vm);
    uint32_t vinc = nv;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(0xffffffffu, vinc, d);
      if (lane >= d) vinc += o;
    }
    const uint32_t vtot = __shfl_sync(0xffffffffu, vinc, 31);
    if (vtot != 0u) {
      uint32_t q = vinc - nv;
      double Sj = S;
#pragma unroll
      for (int j = 0; j < kItems; ++j) {
        if (vm & (1u << j)) {
          cb.sl[q] = Sj;
          cb.i[q] = i0 + j;
          ++q;
        }
        Sj = __dadd_rn(Sj, __dsub_rn(yv[j], c));
      }
      __syncwarp();
      const double Nd = (double)N;
      double bg = -1.0;
      uint32_t bq = 0xffffffffu;
      for (uint32_t e = lane; e < vtot; e += 32) {
        const double sl = cb.sl[e];
        const double g = split_gain_d(sl, sc, (double)cb.i[e], Nd);
        if (g > bg) { bg = g; bq = e; }
      }
      // warp max of the gains, then the lowest index holding it (one redux)
      double g = bg;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) g = fmax(g, __shfl_xor_sync(0xffffffffu, g, off));
      bq = __reduce_min_sync(0xffffffffu, bg == g ? bq : 0xffffffffu);
      best = ArgP{0u, cb.i[bq], g, cb.sl[bq]};  // bq < vtot: gains are >= 0 > -1
      __syncwarp();  // the buffer is rewritten by the next chunk
    }
  }
  if (lane == 0) {
    const uint32_t kf = dsc.k * a.d + dsc.f;
    write_cand(head ? a.head_cand + kf : a.cont_cand + ch, best, kf, a.level, a.slot_gain);
  }
  // node statistics from the feature-0 list (same scan as the general path)
  if (dsc.f == 0) {
    const double v = dsc.v;
    StatP srun{head0 ? 1u : 0u, 0.0, INFINITY, -INFINITY, 0.0};
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
      const double ev = __dsub_rn(yv[j], v);
      srun.sse = __dadd_rn(srun.sse, __dmul_rn(ev, ev));
      srun.ymin = fmin(srun.ymin, yv[j]);
      srun.ymax = fmax(srun.ymax, yv[j]);
      srun.s1 = __dadd_rn(srun.s1, __dsub_rn(yv[j], c));
    }
    StatP st_w;
    const StatP sex = warp_exclusive_scan(srun, StatP{0u, 0.0, INFINITY, -INFINITY, 0.0}, st_w);
    if (lane == 31) {
      StatP ts = srun;
      ts.flag = 0u;
      write_stat(head ? a.head_stat + dsc.k : a.cont_stat + ch, combine(sex, ts));
    }
  }
}

// One pipeline stage of scan_single_kernel: everything one chunk needs, brought in by
// TMA bulk copies (x, y, descriptor, the two carry words, the entry before the chunk).
#ifndef DT_SCAN_STAGES  // experiments: -DDT_SCAN_STAGES=n -DDT_SCAN_MINB=b (DT_EXTRA_NVCC)
#define DT_SCAN_STAGES 2
#endif
#ifndef DT_SCAN_MINB
#define DT_SCAN_MINB 3
#endif
constexpr int kScanStages = DT_SCAN_STAGES;
struct __align__(128) ScanStage {
  float x[kChunkW];
  double y[kChunkW];
  ChunkDesc d;
  SumP cb, ce;   // block carry, chunk-exclusive carry
  float xp[4];   // x[cbase - 4 .. cbase)
  uint32_t ch;
};

// Phase C for the single-segment chunks with a per-warp TMA pipeline: lane 0 keeps
// kScanStages chunks in flight (bulk copies completing on one mbarrier per stage); the
// lanes read their items from shared memory, so no registers hold in-flight data.
__global__ void __launch_bounds__(kThreads, DT_SCAN_MINB) scan_single_kernel(ScanArgs a) {
  extern __shared__ __align__(128) unsigned char scan_smem[];
  const uint32_t K = a.ctl->K[a.parity];
  const uint64_t A = a.ctl->A[a.parity];
  if (K == 0 || A == 0) return;
  const int64_t ns = a.ctl->scnt[0];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  if (gw >= ns) return;  // warp-uniform; no block barriers below
  const uint32_t m = (uint32_t)min(a.min_leaf, (int64_t)0xffffffff);
  ScanStage* st = reinterpret_cast<ScanStage*>(scan_smem) + wib * kScanStages;
  uint64_t* bar = reinterpret_cast<uint64_t*>(scan_smem + sizeof(ScanStage) * kScanStages * (kThreads / 32)) +
                  wib * kScanStages;
  CompactBuf* cbuf = reinterpret_cast<CompactBuf*>(scan_smem + (sizeof(ScanStage) + sizeof(uint64_t)) * kScanStages *
                                                                   (kThreads / 32));
  const bool y32 = a.ctl->y32 != 0;
  const uint32_t ybytes = (uint32_t)(y32 ? sizeof(int32_t) : sizeof(double)) * kChunkW;
  auto issue = [&](int s, int64_t ch) {  // lane 0
    ScanStage& t = st[s];
    t.ch = (uint32_t)ch;
    const uint32_t bytes = (uint32_t)(sizeof(t.x) + sizeof(ChunkDesc) + 2 * sizeof(SumP)) + ybytes +
                           (ch > 0 ? 16u : 0u);
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(bar + s, bytes);
    bulk_g2s(t.x, a.lx + ch * kChunkW, sizeof(t.x), bar + s);
    bulk_g2s(t.y, reinterpret_cast<const char*>(a.ly) + ch * (int64_t)ybytes, ybytes, bar + s);
    bulk_g2s(&t.d, a.desc + ch, sizeof(ChunkDesc), bar + s);
    bulk_g2s(&t.cb, a.block_carry + ch / kBlockChunks, sizeof(SumP), bar + s);
    bulk_g2s(&t.ce, a.chunk_excl + ch, sizeof(SumP), bar + s);
    if (ch > 0) bulk_g2s(t.xp, a.lx + ch * kChunkW - 4, 16, bar + s);
  };
  if (lane == 0) {
    for (int s = 0; s < kScanStages; ++s) mbar_init(bar + s, 1);
    mbar_init_fence();
    for (int s = 0; s < kScanStages; ++s)
      if (gw + s * nw < ns) issue(s, (int64_t)a.list[gw + s * nw]);
  }
  __syncwarp();
  int s = 0;
  uint32_t phase = 0;
  for (int64_t idx = gw; idx < ns; idx += nw) {
    const int64_t nxt = idx + kScanStages * nw;
    const uint32_t ch_ahead = (lane == 0 && nxt < ns) ? a.list[nxt] : 0u;  // consumed after the chunk
    mbar_wait(bar + s, phase);
    const ScanStage& t = st[s];
    float xv[kItems];
    double yv[kItems];
    {
      const float4* x4 = reinterpret_cast<const float4*>(t.x + lane * kItems);
      const double2* y2 = reinterpret_cast<const double2*>(t.y + lane * kItems);
#pragma unroll
      for (int j = 0; j < kItems / 4; ++j) {
        const float4 q = x4[j];
        xv[4 * j] = q.x; xv[4 * j + 1] = q.y; xv[4 * j + 2] = q.z; xv[4 * j + 3] = q.w;
      }
      if (y32) {
        const int4* y4 = reinterpret_cast<const int4*>(reinterpret_cast<const int32_t*>(t.y) + lane * kItems);
#pragma unroll
        for (int j = 0; j < kItems / 4; ++j) {
          const int4 q = y4[j];
          yv[4 * j] = (double)q.x; yv[4 * j + 1] = (double)q.y; yv[4 * j + 2] = (double)q.z; yv[4 * j + 3] = (double)q.w;
        }
      } else {
#pragma unroll
        for (int j = 0; j < kItems / 2; ++j) {
          const double2 q = y2[j];
          yv[2 * j] = q.x; yv[2 * j + 1] = q.y;
        }
      }
    }
    const ChunkDesc dsc = t.d;
    const int64_t ch = t.ch;
    const SumP carry = combine(t.cb, t.ce);
    const float xp0 = t.xp[3];
    __syncwarp();  // every lane has read the stage
    if (lane == 0 && nxt < ns) issue(s, (int64_t)ch_ahead);
    scan_single(a, ch, ch * kChunkW, dsc, xv, yv, m, carry, xp0, cbuf[wib]);
    if (++s == kScanStages) { s = 0; phase ^= 1u; }
  }
}
constexpr size_t kScanSingleSmem =
    (sizeof(ScanStage) + sizeof(uint64_t)) * kScanStages * (kThreads / 32) + sizeof(CompactBuf) * (kThreads / 32);

// Phase C: the main scan (prefixes, gains, per-piece argmax, node statistics), one warp
// chunk at a time per warp, no block barriers.
#ifndef DT_SCANK_MINB
#define DT_SCANK_MINB 2
#endif
__global__ void __launch_bounds__(kThreads, DT_SCANK_MINB) scan_kernel(ScanArgs a) {
  // per-thread best of the run before its first head (written and read by the same
  // thread, so no barrier is needed)
  __shared__ double fr_gain[kThreads], fr_sl[kThreads], fs_sse[kThreads], fs_min[kThreads],
      fs_max[kThreads], fs_s1[kThreads];
  __shared__ uint32_t fr_i[kThreads];

  const uint32_t K = a.ctl->K[a.parity];
  const uint64_t A = a.ctl->A[a.parity];
  if (K == 0 || A == 0) return;
  const int64_t total = (int64_t)A * a.dl;
  const int64_t nch = (total + kChunkW - 1) / kChunkW;
  const int tid = threadIdx.x, lane = tid & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const uint32_t m = (uint32_t)min(a.min_leaf, (int64_t)0xffffffff);
  const SumP sum0{0u, 0.0};
  const ArgP arg0{0u, 0xffffffffu, -1.0, 0.0};
  const StatP stat0{0u, 0.0, INFINITY, -INFINITY, 0.0};

  // the chunks with a segment boundary inside (list tail); register double buffering:
  // the next chunk's loads are in flight during this chunk
  const int64_t ng = a.ctl->scnt[1];
  float xn[kItems];
  double yn[kItems];
  const bool y32 = a.ctl->y32 != 0;
  int64_t ch_next = (gw < ng) ? (int64_t)a.list[nch - 1 - gw] : 0;
  {
    const int64_t q0 = ch_next * kChunkW + lane * kItems;
    if (gw < ng && q0 < total) load_items(a.lx, a.ly, q0, total, xn, yn, y32);
  }
  for (int64_t idx = gw; idx < ng; idx += nw) {
    const int64_t ch = ch_next;
    const int64_t p0 = ch * kChunkW + lane * kItems;
    const bool any = p0 < total;
    float xv[kItems];
    double yv[kItems];
#pragma unroll
    for (int j = 0; j < kItems; ++j) { xv[j] = xn[j]; yv[j] = yn[j]; }
    if (idx + nw < ng) {
      ch_next = (int64_t)a.list[nch - 1 - (idx + nw)];
      const int64_t q0 = ch_next * kChunkW + lane * kItems;
      if (q0 < total) load_items(a.lx, a.ly, q0, total, xn, yn, y32);
    }
    const ChunkDesc dsc = a.desc[ch];
    Seg sg{0, 0, 0, 0u, 0};
    if (any) seg_from(sg, dsc.start, dsc.end, dsc.k, dsc.f, A, p0, a.nodes, K);
    // Warp-uniform fast path: every lane's kItems entries lie in ONE segment (a head may
    // only sit at its item 0).  True for nearly all warps at shallow levels.
    const bool one_seg = any && (p0 + kItems <= total) && (sg.end >= p0 + kItems);
    const bool warp_fast = __all_sync(0xffffffffu, one_seg || !any);
    const bool head0 = any && (p0 == sg.start);
    // node fields of my first segment: from the descriptor when it is the chunk's segment
    const bool in_d = (sg.k == dsc.k && sg.f == dsc.f);
    const double nd_c = in_d ? dsc.c : __ldg(&a.nodes[sg.k].c);
    const SumP tagg = thread_sum_agg(a, K, A, p0, total, any, warp_fast, head0, sg, yv, nd_c);
    SumP wagg;
    const SumP texcl = warp_exclusive_scan(tagg, sum0, wagg);
    const SumP carry = combine(a.block_carry[ch / kBlockChunks], a.chunk_excl[ch]);
    double S = combine(carry, texcl).s;  // exclusive prefix at my item 0

    // ---- pass 2: prefixes, gains, per-run best; flush runs that end in this thread
    ArgP run = arg0;
    bool seen_head = false;
    int last_f = sg.f;
    uint32_t last_k = sg.k;
    const bool stats_tile = (ch * kChunkW) < (int64_t)A;  // chunk holds feature-0 items
    if (any && warp_fast) {
      if (head0) {
        fr_gain[tid] = -1.0; fr_sl[tid] = 0.0; fr_i[tid] = 0xffffffffu;
        seen_head = true;
        run.flag = 1u;
        S = 0.0;
      }
      if (in_d ? dsc.srch : __ldg(&a.nodes[sg.k].searchable)) {
        const double c = nd_c, sc = in_d ? dsc.sc : __ldg(&a.nodes[sg.k].sc);
        const uint32_t N = in_d ? dsc.N : __ldg(&a.nodes[sg.k].N);
        const uint32_t i0 = (uint32_t)(p0 - sg.start);
        const uint32_t ilo = m > 1u ? m : 1u, ihi = N - m;
        const float xprev = head0 ? 0.f : a.lx[p0 - 1];
        const double Nd = (double)N, nl0 = (double)i0;
        // loop 1: approximate gains (exact D and denominator, reciprocal by Newton)
        double Sj = S, bapx = -1.0, bS = 0.0;
        int bj = -1;
        bool amb = false;
        constexpr double kTol = 1e-13;  // >> |approx - exact| / exact (~3e-16)
#pragma unroll
        for (int j = 0; j < kItems; ++j) {
          const uint32_t i = i0 + j;
          const float xp = (j == 0) ? xprev : xv[j - 1];
          if (i >= ilo && i <= ihi && xp < xv[j]) {
            const double g = split_gain_approx_d(Sj, sc, __dadd_rn(nl0, (double)j), Nd);
            if (g > bapx) {
              if (bapx >= __dmul_rn(g, 1.0 - kTol)) amb = true;
              bapx = g; bS = Sj; bj = j;
            } else if (g >= __dmul_rn(bapx, 1.0 - kTol)) {
              amb = true;
            }
          }
          Sj = __dadd_rn(Sj, __dsub_rn(yv[j], c));
        }
        if (bj >= 0 && !amb) {
          // the exact argmax is the approximate one: exact gain of that position only
          const uint32_t i = i0 + (uint32_t)bj;
          run.gain = split_gain_d(bS, sc, __dadd_rn(nl0, (double)bj), Nd);
          run.i = i;
          run.sl = bS;
        } else if (bj >= 0) {
          // near-tie: exact gains at every valid position (strict >, position order)
          Sj = S;
#pragma unroll
          for (int j = 0; j < kItems; ++j) {
            const uint32_t i = i0 + j;
            const float xp = (j == 0) ? xprev : xv[j - 1];
            if (i >= ilo && i <= ihi && xp < xv[j]) {
              const double g = split_gain_d(Sj, sc, __dadd_rn(nl0, (double)j), Nd);
              if (g > run.gain) { run.gain = g; run.i = i; run.sl = Sj; }
            }
            Sj = __dadd_rn(Sj, __dsub_rn(yv[j], c));
          }
        }
      }
    } else if (any) {
      Seg s = sg;
      double nc = __ldg(&a.nodes[s.k].c), nsc = __ldg(&a.nodes[s.k].sc);
      uint32_t nN = __ldg(&a.nodes[s.k].N);
      int nsrch = __ldg(&a.nodes[s.k].searchable);
      float xprev = (p0 > sg.start) ? a.lx[p0 - 1] : 0.f;
#pragma unroll
      for (int j = 0; j < kItems; ++j) {
        const int64_t p = p0 + j;
        if (p < total) {
          if (p == s.end) {
            seg_next(s, a.nodes, K, A);
            nc = __ldg(&a.nodes[s.k].c);
            nsc = __ldg(&a.nodes[s.k].sc);
            nN = __ldg(&a.nodes[s.k].N);
            nsrch = __ldg(&a.nodes[s.k].searchable);
          }
          if (p == s.start) {
            if (!seen_head) {
              fr_gain[tid] = run.gain; fr_sl[tid] = run.sl; fr_i[tid] = run.i;
            } else {
              // the previous run is a whole segment that started in this thread
              const int pf = (s.k == 0) ? s.f - 1 : s.f;
              const uint32_t pk = (s.k == 0) ? (K - 1) : s.k - 1;
              write_cand(a.head_cand + (int64_t)pk * a.d + pf, run, pk * a.d + pf, a.level, a.slot_gain);
            }
            seen_head = true;
            run = arg0;
            run.flag = 1u;
            S = 0.0;
          }
          const uint32_t i = (uint32_t)(p - s.start);
          if (nsrch && i >= 1 && i >= m && nN - i >= m) {
            const float xp = (j == 0) ? xprev : xv[j - 1];
            if (xp < xv[j]) {
              const double g = split_gain(S, nsc, i, nN);
              if (g > run.gain) { run.gain = g; run.i = i; run.sl = S; }
            }
          }
          S = __dadd_rn(S, __dsub_rn(yv[j], nc));
          last_f = s.f;
          last_k = s.k;
        }
      }
    }
    // ---- node statistics (feature-0 tiles only): sum (y - v)^2, min, max, sum (y - c)
    StatP srun = stat0;
    if (stats_tile && any) {
      Seg s = sg;
      double nc = __ldg(&a.nodes[s.k].c), nv = __ldg(&a.nodes[s.k].v);
      bool seen = false;
#pragma unroll
      for (int j = 0; j < kItems; ++j) {
        const int64_t p = p0 + j;
        if (p < total) {
          if (p == s.end) {
            seg_next(s, a.nodes, K, A);
            nc = __ldg(&a.nodes[s.k].c);
            nv = __ldg(&a.nodes[s.k].v);
          }
          if (p == s.start) {
            if (!seen) {
              fs_sse[tid] = srun.sse; fs_min[tid] = srun.ymin; fs_max[tid] = srun.ymax;
              fs_s1[tid] = srun.s1;
            } else {
              const int pf = (s.k == 0) ? s.f - 1 : s.f;
              const uint32_t pk = (s.k == 0) ? (K - 1) : s.k - 1;
              if (pf == 0) write_stat(a.head_stat + pk, srun);
            }
            seen = true;
            srun = stat0;
            srun.flag = 1u;
          }
          if (s.f == 0) {
            const double ev = __dsub_rn(yv[j], nv);
            srun.sse = __dadd_rn(srun.sse, __dmul_rn(ev, ev));
            srun.ymin = fmin(srun.ymin, yv[j]);
            srun.ymax = fmax(srun.ymax, yv[j]);
            srun.s1 = __dadd_rn(srun.s1, __dsub_rn(yv[j], nc));
          }
        }
      }
    }
    ArgP trail = run;
    trail.flag = seen_head ? 1u : 0u;
    StatP strail = srun;
    strail.flag = seen_head ? 1u : 0u;

    ArgP arg_w;
    const ArgP aex = warp_exclusive_scan(trail, arg0, arg_w);
    StatP sex = stat0, st_w;
    if (stats_tile) sex = warp_exclusive_scan(strail, stat0, st_w);

    // Flush the open segment that ends at my first head (its earlier part is in aex).
    if (any && seen_head) {
      const bool item0_head = (p0 == sg.start);
      if (!(lane == 0 && item0_head)) {
        int of;
        uint32_t ok;
        if (!item0_head) { of = sg.f; ok = sg.k; }
        else if (sg.k > 0) { of = sg.f; ok = sg.k - 1; }
        else { of = sg.f - 1; ok = K - 1; }
        const ArgP fr{0u, fr_i[tid], fr_gain[tid], fr_sl[tid]};
        const ArgP done_a = combine(aex, fr);
        const bool head_in_chunk = aex.flag != 0;
        const uint32_t kf = ok * a.d + of;
        if (head_in_chunk) write_cand(a.head_cand + kf, done_a, kf, a.level, a.slot_gain);
        else write_cand(a.cont_cand + ch, done_a, kf, a.level, a.slot_gain);
        if (stats_tile && of == 0) {
          const StatP fs{0u, fs_sse[tid], fs_min[tid], fs_max[tid], fs_s1[tid]};
          const StatP done_s = combine(sex, fs);
          if (head_in_chunk) write_stat(a.head_stat + ok, done_s);
          else write_stat(a.cont_stat + ch, done_s);
        }
      }
    }
    // The last lane closes the segment open at the chunk end.
    if (lane == 31) {
      uint32_t lk = last_k;
      int lff = last_f;
      if (!any) {
        Seg t;
        seg_from(t, dsc.start, dsc.end, dsc.k, dsc.f, A, min(total, ch * kChunkW + kChunkW) - 1, a.nodes, K);
        lk = t.k;
        lff = t.f;
      }
      ArgP tr = run;
      tr.flag = 0u;
      const ArgP done_a = seen_head ? run : combine(aex, tr);
      const bool head_in_chunk = seen_head || aex.flag != 0;
      const uint32_t kf = lk * a.d + lff;
      if (head_in_chunk) write_cand(a.head_cand + kf, done_a, kf, a.level, a.slot_gain);
      else write_cand(a.cont_cand + ch, done_a, kf, a.level, a.slot_gain);
      if (stats_tile && lff == 0) {
        StatP ts = srun;
        ts.flag = 0u;
        const StatP done_s = seen_head ? srun : combine(sex, ts);
        if (head_in_chunk) write_stat(a.head_stat + lk, done_s);
        else write_stat(a.cont_stat + ch, done_s);
      }
    }
  }
}

// Lowest position among the pieces of each segment whose gain equals the segment max.
__global__ void __launch_bounds__(256) piece_pos_kernel(ScanArgs a, uint32_t* __restrict__ slot_pos) {
  const uint32_t K = a.ctl->K[a.parity];
  const uint64_t A = a.ctl->A[a.parity];
  if (K == 0 || A == 0) return;
  const int64_t total = (int64_t)A * a.dl;
  const int64_t nch = (total + kChunkW - 1) / kChunkW;
  const int64_t nhead = (int64_t)K * a.d;
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < nch + nhead;
       r += (int64_t)gridDim.x * blockDim.x) {
    const Cand c = (r < nch) ? a.cont_cand[r] : a.head_cand[r - nch];
    if (c.level != a.level || !(c.gain >= 0.0) || (int64_t)c.kf >= nhead) continue;
    if ((unsigned long long)__double_as_longlong(c.gain) == a.slot_gain[c.kf]) atomicMin(slot_pos + c.kf, c.i);
  }
}

// ----------------------------------------------------------------------------- select --

struct SelectArgs {
  uint4* gbits;  // go-left bitmap: zeroed here (grid-stride) for this level's prep_kernel
  int64_t nvec;
  const float* lx;
  const NodeL* nodes;
  Ctl* ctl;
  int parity;
  int level;
  int dl;
  int d;
  const Cand* head_cand;
  const Cand* cont_cand;
  const Stat* head_stat;
  const Stat* cont_stat;
  Decision* dec;
  dt_node* out;
  LevelLog* log;
  unsigned long long* slot_gain;
  uint32_t* slot_pos;
  ExchRec* exch;       // [K] this rank's records
  int world, rank, dg;  // feature sharding: local feature j is global j * world + rank
};

// Leaf rules and the decision of node k from the ranks' records (see decide_kernel).
__device__ __forceinline__ void decide_node(const SelectArgs& a, uint32_t k, const NodeL& nd,
                                            const ExchRec* __restrict__ all, int64_t stride) {
  const ExchRec st = all[k];  // rank 0
  const bool pure = !(st.ymin < st.ymax);
  int bf = -1;
  ExchRec best;
  best.gain = -1.0;
  if (nd.searchable && !pure) {
    for (int r = 0; r < a.world; ++r) {
      const ExchRec c = all[(int64_t)r * stride + k];
      if (c.gain < 0.0) continue;
      if (bf < 0 || c.gain > best.gain || (c.gain == best.gain && c.gf < bf)) {
        best = c;
        bf = c.gf;
      }
    }
    atomicAdd(&a.ctl->split_evals, (unsigned long long)nd.N * (unsigned long long)a.dg);
  }
  Decision dc;
  dt_node o;
  o.depth = a.level;
  // value = mean of the node's own rows.  Integer mode: exact fl(S/N) from the exact
  // bookkeeping.  Real mode: centre + fresh sum (y - c) / N, and exactly y for a pure
  // node (all rows equal), so single-row leaves reproduce their target.
  if (a.ctl->int_mode) o.value = nd.v;
  else o.value = pure ? st.ymin : __dadd_rn(nd.c, __ddiv_rn(st.s1, (double)nd.N));
  o.impurity = __ddiv_rn(st.sse, (double)nd.N);
  o.n_samples = nd.N;
  o.left = -1;
  o.right = -1;
  dc.pad = 0;
  if (bf >= 0) {
    dc.f = bf;
    dc.floc = (bf % a.world == a.rank) ? bf / a.world : -1;
    dc.nl = best.i;
    dc.sl = best.sl;
    dc.thr = best.thr;
    o.feature = bf;
    o.threshold = best.thr;
  } else {
    dc.f = -1;
    dc.floc = -1;
    dc.nl = 0;
    dc.sl = 0.0;
    dc.thr = 0.0;
    o.feature = -1;
    o.threshold = 0.0;
  }
  a.dec[k] = dc;
  a.out[nd.id] = o;
  atomicMax(&a.ctl->max_depth_seen, a.level);
}

// Folds the node-statistics pieces [lo, hi) of node k in index order: loads issued in
// batches of 8 ahead of the (sequential, order-preserving) combination, so a long run
// costs one memory latency per 8 pieces instead of one per piece.
__device__ __forceinline__ void fold_stats(const SelectArgs& a, uint32_t k, int64_t t0, int64_t lo, int64_t hi,
                                           Stat& acc) {
  for (int64_t b = lo; b < hi; b += 8) {
    Stat v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int64_t pc = b + u;
      if (pc < hi) v[u] = (pc == 0) ? a.head_stat[k] : a.cont_stat[t0 + pc];
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      if (b + u < hi) {
        acc.sse = __dadd_rn(acc.sse, v[u].sse);
        acc.ymin = fmin(acc.ymin, v[u].ymin);
        acc.ymax = fmax(acc.ymax, v[u].ymax);
        acc.s1 = __dadd_rn(acc.s1, v[u].s1);
      }
    }
  }
}

// One block per node (grid-stride over the level's nodes).
#ifndef DT_SEL_MINB
#define DT_SEL_MINB 1
#endif
__global__ void __launch_bounds__(256, DT_SEL_MINB) select_kernel(SelectArgs a) {
  const uint32_t K = a.ctl->K[a.parity];
  const uint64_t A = a.ctl->A[a.parity];
  __shared__ double s_gain[256];
  __shared__ uint32_t s_i[256];
  __shared__ double s_sl[256];
  __shared__ Stat s_stat[256];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  // nothing reads the bitmap between the previous level's partition and this level's
  // prep_kernel; clearing it here spreads the 128 KB (C2) / 12.5 MB (C3) over the whole
  // grid instead of number_kernel's single block
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + tid; i < a.nvec; i += (int64_t)gridDim.x * blockDim.x)
    a.gbits[i] = make_uint4(0u, 0u, 0u, 0u);
  if (blockIdx.x == 0 && tid == 0 && a.level < kMaxLogLevels) {
    a.log[a.level].A = A;
    a.log[a.level].K = K;
    a.log[a.level].A_next = 0;
    a.log[a.level].K_next = 0;
  }
  if (K > gridDim.x) {
    // Many (small) nodes: one warp per node, no block barriers.  Same per-feature bests;
    // node statistics by a fixed-shape warp reduction (contiguous runs of pieces per lane,
    // then an xor tree); the feature argmax keeps the lowest feature among equal gains.
    const int nwarps = blockDim.x >> 5;
    for (uint32_t k = blockIdx.x * nwarps + w; k < K; k += gridDim.x * nwarps) {
      const NodeL nd = a.nodes[k];
      double bg = -1.0, bsl = 0.0;
      uint32_t bi = 0xffffffffu;
      int bf = 0x7fffffff;
      for (int f = lane; f < a.d; f += 32) {
        const uint32_t kf = k * a.d + f;
        if (nd.searchable && f < a.dl && nd.N > 1) {
          const uint32_t pos = a.slot_pos[kf];
          if (pos != 0xffffffffu) {
            const double g = __longlong_as_double((long long)a.slot_gain[kf]);
            if (g > bg) {  // strict >: the lowest of this lane's features wins ties
              const int64_t s0 = (int64_t)f * (int64_t)A + nd.start;
              const int64_t t0 = s0 / kChunkW, c = (s0 + pos) / kChunkW;
              bsl = ((c == t0) ? a.head_cand[kf] : a.cont_cand[c]).sl;
              bg = g;
              bi = pos;
              bf = f;
            }
          }
        }
        a.slot_gain[kf] = 0ull;
        a.slot_pos[kf] = 0xffffffffu;
      }
      double gmax = bg;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) gmax = fmax(gmax, __shfl_xor_sync(0xffffffffu, gmax, off));
      const int wf = __reduce_min_sync(0xffffffffu, (bg == gmax && bg >= 0.0) ? bf : 0x7fffffff);
      const int src = __ffs(__ballot_sync(0xffffffffu, bf == wf)) - 1;
      const uint32_t wi = __shfl_sync(0xffffffffu, bi, src < 0 ? 0 : src);
      const double wsl = __shfl_sync(0xffffffffu, bsl, src < 0 ? 0 : src);
      // node statistics from the feature-0 list
      const int64_t s0 = nd.start, s1 = s0 + nd.N - 1;
      const int64_t t0 = s0 / kChunkW, t1 = s1 / kChunkW;
      const int64_t np = t1 - t0 + 1;
      const int64_t per = (np + 31) / 32;
      Stat acc{0.0, INFINITY, -INFINITY, 0.0};
      fold_stats(a, k, t0, lane * per, min(np, (lane + 1) * per), acc);
#pragma unroll
      for (int off = 1; off < 32; off <<= 1) {  // lane l absorbs lane l + off (fixed shape)
        const double o_sse = __shfl_down_sync(0xffffffffu, acc.sse, off);
        const double o_min = __shfl_down_sync(0xffffffffu, acc.ymin, off);
        const double o_max = __shfl_down_sync(0xffffffffu, acc.ymax, off);
        const double o_s1 = __shfl_down_sync(0xffffffffu, acc.s1, off);
        if ((lane & (2 * off - 1)) == 0) {
          acc.sse = __dadd_rn(acc.sse, o_sse);
          acc.ymin = fmin(acc.ymin, o_min);
          acc.ymax = fmax(acc.ymax, o_max);
          acc.s1 = __dadd_rn(acc.s1, o_s1);
        }
      }
      if (lane == 0) {
        ExchRec r;
        r.gain = -1.0;
        r.sl = 0.0;
        r.thr = 0.0;
        r.i = 0;
        r.gf = -1;
        if (wf != 0x7fffffff) {
          const int64_t pos = (int64_t)wf * (int64_t)A + nd.start + wi;
          const double xlo = (double)a.lx[pos - 1], xhi = (double)a.lx[pos];
          r.gain = gmax;
          r.sl = wsl;
          r.i = wi;
          r.gf = wf * a.world + a.rank;
          r.thr = __dadd_rn(__ddiv_rn(xlo, 2.0), __ddiv_rn(xhi, 2.0));  // Reading R5
        }
        r.sse = acc.sse;
        r.ymin = acc.ymin;
        r.ymax = acc.ymax;
        r.s1 = acc.s1;
        a.exch[k] = r;
        if (a.world == 1) decide_node(a, k, nd, a.exch, 0);  // single rank: decide in place
      }
    }
    return;
  }
  for (uint32_t k = blockIdx.x; k < K; k += gridDim.x) {
    const NodeL nd = a.nodes[k];
    // ---- per-feature best: max gain (slot_gain) at the lowest position (slot_pos); the
    // winner's S'_L comes from the piece record that holds that position.  Slots are reset.
    for (int f = tid; f < a.d; f += blockDim.x) {
      double bg = -1.0, bsl = 0.0;
      uint32_t bi = 0xffffffffu;
      const uint32_t kf = k * a.d + f;
      if (nd.searchable && f < a.dl && nd.N > 1) {
        const uint32_t pos = a.slot_pos[kf];
        if (pos != 0xffffffffu) {
          const int64_t s0 = (int64_t)f * (int64_t)A + nd.start;
          const int64_t t0 = s0 / kChunkW, c = (s0 + pos) / kChunkW;
          const Cand rec = (c == t0) ? a.head_cand[kf] : a.cont_cand[c];
          bg = __longlong_as_double((long long)a.slot_gain[kf]);
          bi = pos;
          bsl = rec.sl;
        }
      }
      a.slot_gain[kf] = 0ull;
      a.slot_pos[kf] = 0xffffffffu;
      s_gain[f] = bg; s_i[f] = bi; s_sl[f] = bsl;
    }
    __syncthreads();
    // ---- node statistics from the feature-0 list (fixed-shape reduction)
    {
      const int64_t s0 = nd.start, s1 = s0 + nd.N - 1;
      const int64_t t0 = s0 / kChunkW, t1 = s1 / kChunkW;
      Stat acc{0.0, INFINITY, -INFINITY, 0.0};  // s1 accumulates sum (y - c)
      // each thread folds a contiguous run of pieces, then tree
      const int64_t np = t1 - t0 + 1;
      const int64_t per = (np + blockDim.x - 1) / blockDim.x;
      fold_stats(a, k, t0, tid * per, min(np, (tid + 1) * per), acc);
      s_stat[tid] = acc;
      __syncthreads();
      for (int off = 128; off > 0; off >>= 1) {
        if (tid < off) {
          Stat& x = s_stat[tid];
          const Stat y = s_stat[tid + off];
          x.sse = __dadd_rn(x.sse, y.sse);
          x.ymin = fmin(x.ymin, y.ymin);
          x.ymax = fmax(x.ymax, y.ymax);
          x.s1 = __dadd_rn(x.s1, y.s1);
        }
        __syncthreads();
      }
    }
    if (tid == 0) {
      const Stat st = s_stat[0];
      int bf = -1;
      double bg = -1.0, bsl = 0.0;
      uint32_t bi = 0;
      for (int f = 0; f < a.d; ++f)
        if (s_gain[f] > bg) { bg = s_gain[f]; bi = s_i[f]; bsl = s_sl[f]; bf = f; }  // strict >
      ExchRec r;
      r.gain = -1.0;
      r.sl = 0.0;
      r.thr = 0.0;
      r.i = 0;
      r.gf = -1;
      if (bf >= 0 && bg >= 0.0) {
        const int64_t pos = (int64_t)bf * (int64_t)A + nd.start + bi;
        const double xlo = (double)a.lx[pos - 1], xhi = (double)a.lx[pos];
        r.gain = bg;
        r.sl = bsl;
        r.i = bi;
        r.gf = bf * a.world + a.rank;
        r.thr = __dadd_rn(__ddiv_rn(xlo, 2.0), __ddiv_rn(xhi, 2.0));  // Reading R5
      }
      r.sse = st.sse;
      r.ymin = st.ymin;
      r.ymax = st.ymax;
      r.s1 = st.s1;
      a.exch[k] = r;
      if (a.world == 1) decide_node(a, k, nd, a.exch, 0);  // single rank: decide in place
    }
    __syncthreads();
  }
}

// Combines the ranks' records of every node (fixed order: highest gain, then lowest
// global feature, Reading R4; statistics from rank 0, which owns feature 0) and applies
// the leaf rules (Reading R8).  Identical inputs on every rank -> identical trees.
__global__ void __launch_bounds__(256) decide_kernel(SelectArgs a, const ExchRec* __restrict__ all,
                                                     int64_t stride) {
  const uint32_t K = a.ctl->K[a.parity];
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < K; k += gridDim.x * blockDim.x)
    decide_node(a, k, a.nodes[k], all, stride);
}

// ----------------------------------------------------------------------------- number --

struct NumberArgs {
  const NodeL* nodes;
  NodeL* next;
  const Decision* dec;
  uint32_t* new_start;  // [K] left-child start in the next lists (or 0xffffffff)
  Ctl* ctl;
  int parity;
  int level;
  int32_t max_depth;
  int64_t min_leaf;
  dt_node* out;
  LevelLog* log;
};

// Single block: BFS numbering (children appended left, right in node order), child
// statistics, next-level offsets.  Integer mode keeps every quantity exact (int64).
__global__ void __launch_bounds__(1024) number_kernel(NumberArgs a) {
  __shared__ CntP sh[33];
  __shared__ unsigned long long sh_rows[33];
  __shared__ uint32_t base_split;
  __shared__ unsigned long long base_rows;
  const uint32_t K = a.ctl->K[a.parity];
  const int tid = threadIdx.x;
  const int next_id0 = a.ctl->next_id;
  const int int_mode = a.ctl->int_mode;
  if (tid == 0) { base_split = 0; base_rows = 0; }
  __syncthreads();
  for (uint32_t k0 = 0; k0 < K; k0 += blockDim.x) {
    const uint32_t k = k0 + tid;
    const bool in = k < K;
    const Decision dc = in ? a.dec[k] : Decision{-1, 0, 0.0, 0.0};
    const bool sp = in && dc.f >= 0;
    const NodeL nd = in ? a.nodes[k] : NodeL{};
    CntP agg;
    CntP ex = block_exclusive_scan(CntP{0u, sp ? 1u : 0u}, CntP{0u, 0u}, agg, sh);
    // exclusive scan of rows of split nodes (64-bit, via warp shuffles)
    unsigned long long rv = sp ? nd.N : 0ull, inc = rv;
    const int lane = tid & 31, w = tid >> 5;
    for (int dd = 1; dd < 32; dd <<= 1) {
      unsigned long long o = __shfl_up_sync(0xffffffffu, inc, dd);
      if (lane >= dd) inc += o;
    }
    if (lane == 31) sh_rows[w] = inc;
    __syncthreads();
    if (tid == 0) {
      unsigned long long run = 0;
      for (int i = 0; i < (int)(blockDim.x >> 5); ++i) { unsigned long long t = sh_rows[i]; sh_rows[i] = run; run += t; }
      sh_rows[32] = run;
    }
    __syncthreads();
    const unsigned long long rows_ex = base_rows + sh_rows[w] + (inc - rv);
    const uint32_t rank = base_split + ex.c;
    if (in) {
      if (sp) {
        const int lid = next_id0 + 2 * (int)rank;
        a.out[nd.id].left = lid;
        a.out[nd.id].right = lid + 1;
        a.new_start[k] = (uint32_t)rows_ex;
        const uint32_t nl = dc.nl, nr = nd.N - dc.nl;
        NodeL L, R;
        L.start = (uint32_t)rows_ex;
        L.N = nl;
        L.id = lid;
        R.start = (uint32_t)rows_ex + nl;
        R.N = nr;
        R.id = lid + 1;
        const int child_depth = a.level + 1;
        const bool depth_ok = (a.max_depth < 0) || (child_depth < a.max_depth);
        L.searchable = (depth_ok && (int64_t)nl >= 2 * a.min_leaf) ? 1 : 0;
        R.searchable = (depth_ok && (int64_t)nr >= 2 * a.min_leaf) ? 1 : 0;
        L.pad = R.pad = 0.0;
        const double slp = dc.sl;                    // parent-centred S'_L
        const double srp = __dsub_rn(nd.sc, slp);    // parent-centred S'_R
        if (int_mode) {
          const long long cp = (long long)nd.c;
          const long long SL = (long long)nl * cp + (long long)slp;
          const long long SR = (long long)nr * cp + (long long)srp;
          const long long cl = floor_div_ll(SL, nl), cr = floor_div_ll(SR, nr);
          L.c = (double)cl;
          R.c = (double)cr;
          L.v = __ddiv_rn((double)SL, (double)nl);
          R.v = __ddiv_rn((double)SR, (double)nr);
          L.sc = (double)(SL - (long long)nl * cl);
          R.sc = (double)(SR - (long long)nr * cr);
        } else {
          L.v = __dadd_rn(nd.c, __ddiv_rn(slp, (double)nl));
          R.v = __dadd_rn(nd.c, __ddiv_rn(srp, (double)nr));
          L.c = L.v;
          R.c = R.v;
          // re-centre: S'_child = S'_(parent-centred) - n * (c_child - c_parent)
          L.sc = __dsub_rn(slp, __dmul_rn((double)nl, __dsub_rn(L.c, nd.c)));
          R.sc = __dsub_rn(srp, __dmul_rn((double)nr, __dsub_rn(R.c, nd.c)));
        }
        a.next[2 * rank] = L;
        a.next[2 * rank + 1] = R;
      } else {
        a.new_start[k] = 0xffffffffu;
      }
    }
    __syncthreads();
    if (tid == 0) { base_split += agg.c; base_rows += sh_rows[32]; }
    __syncthreads();
  }
  if (tid == 0) {
    const int np = a.parity ^ 1;
    a.ctl->pcnt[0] = a.ctl->pcnt[1] = 0;  // this level's partition lists (prep_kernel)
    a.ctl->scnt[0] = a.ctl->scnt[1] = 0;  // the next level's scan lists (prep_kernel)
    a.ctl->K[np] = 2 * base_split;
    a.ctl->A[np] = base_rows;
    a.ctl->next_id = next_id0 + 2 * (int)base_split;
    if (a.level < kMaxLogLevels) {
      a.log[a.level].A_next = base_rows;
      a.log[a.level].K_next = 2 * base_split;
    }
  }
}

// ----------------------------------------------------------------------------- goleft --

// ----------------------------------------------------------------------------- partition --

// Binary search over a level's node starts cached in shared memory: largest k with
// st[k] <= q.
__device__ __forceinline__ uint32_t find_start(const uint32_t* st, uint32_t K, uint32_t q) {
  uint32_t lo = 0, hi = K;
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (st[mid] <= q) lo = mid; else hi = mid;
  }
  return lo;
}

struct PrepArgs {
  const uint32_t* lr;         // this level's row lists
  const NodeL* nodes;         // this level's nodes
  const NodeL* next;          // next level's nodes (from number_kernel)
  const Decision* dec;
  const uint32_t* new_start;
  uint32_t* gbits;            // go-left bitmap (zeroed by select_kernel)
  PartDesc* pdesc;
  uint32_t* plist;
  ChunkDesc* sdesc;
  uint32_t* slist;
  Ctl* ctl;
  int parity;
  int dl_out;   // lists the partition writes (= lists the next level scans)
};
constexpr int kPrepCache = 12288;  // node starts of both levels cached per block (48 KB)
#ifndef DT_PREP_THREADS
#define DT_PREP_THREADS 1024
#endif
constexpr int kPrepThreads = DT_PREP_THREADS;

// Everything between the numbering of level l and its partition, in one launch (one
// block per SM, the node starts of levels l and l+1 in shared memory):
//   goleft:    bit per row of every split node's left rows (a6);
//   part desc: level-l partition chunk descriptors and chunk lists;
//   scan desc: level-(l+1) scan chunk descriptors and chunk lists.
// The three index spaces are independent; the list counters were reset by number_kernel.
__global__ void __launch_bounds__(kPrepThreads) prep_kernel(PrepArgs a) {
  __shared__ uint32_t st[kPrepCache];
  const uint32_t K = a.ctl->K[a.parity], K2 = a.ctl->K[a.parity ^ 1];
  const uint64_t A = a.ctl->A[a.parity], A2 = a.ctl->A[a.parity ^ 1];
  if (K == 0 || A == 0 || A2 == 0) return;  // nothing splits: nothing moves, no next level
  const bool cache = (uint64_t)K + K2 <= (uint64_t)kPrepCache;
  uint32_t* s1 = st;
  uint32_t* s2 = st + K;
  if (cache) {
    for (uint32_t i = threadIdx.x; i < K; i += blockDim.x) s1[i] = __ldg(&a.nodes[i].start);
    for (uint32_t i = threadIdx.x; i < K2; i += blockDim.x) s2[i] = __ldg(&a.next[i].start);
    __syncthreads();
  }
  constexpr int kI = 8;  // goleft positions per work item
  const int64_t G = ((int64_t)A + kI - 1) / kI;
  const int64_t P = ((int64_t)A * a.dl_out + kChunkW - 1) / kChunkW;
  const int64_t S = ((int64_t)A2 * a.dl_out + kChunkW - 1) / kChunkW;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < G + P + S;
       t += (int64_t)gridDim.x * blockDim.x) {
    if (t < G) {
      // positions q0 .. q0 + kI - 1 of the split features' lists: all row loads first
      // (independent), then the bit atomics
      const uint32_t q0 = (uint32_t)(t * kI);
      uint32_t k = cache ? find_start(s1, K, q0) : find_node(a.nodes, K, q0);
      uint32_t kstart = __ldg(&a.nodes[k].start), kend = kstart + __ldg(&a.nodes[k].N);
      int32_t floc = __ldg(&a.dec[k].floc);
      uint32_t nl = __ldg(&a.dec[k].nl);
      uint32_t rr[kI];
      bool go[kI];
#pragma unroll
      for (int j = 0; j < kI; ++j) {
        const uint32_t q = q0 + j;
        go[j] = false;
        if ((uint64_t)q < A) {
          while (q >= kend) {
            ++k;
            kstart = kend;
            kend = kstart + __ldg(&a.nodes[k].N);
            floc = __ldg(&a.dec[k].floc);
            nl = __ldg(&a.dec[k].nl);
          }
          go[j] = floc >= 0 && q - kstart < nl;
          rr[j] = go[j] ? __ldg(&a.lr[(int64_t)floc * (int64_t)A + q]) : 0u;
        }
      }
#pragma unroll
      for (int j = 0; j < kI; ++j)
        if (go[j]) atomicOr(a.gbits + (rr[j] >> 5), 1u << (rr[j] & 31));
    } else if (t < G + P) {
      const int64_t c = t - G;
      const int64_t p = c * kChunkW;
      const int f = (int)(p / (int64_t)A);
      const int64_t fbase = (int64_t)f * (int64_t)A;
      const uint32_t q = (uint32_t)(p - fbase);
      const uint32_t k = cache ? find_start(s1, K, q) : find_node(a.nodes, K, q);
      PartDesc d;
      d.start = fbase + __ldg(&a.nodes[k].start);
      d.end = d.start + __ldg(&a.nodes[k].N);
      d.k = k;
      d.f = f;
      const Decision dc = a.dec[k];
      d.nl = dc.nl;
      d.split = dc.f >= 0 ? 1 : 0;
      d.ns = __ldg(&a.new_start[k]);
      d.pad = 0;
      a.pdesc[c] = d;
      // single-segment chunks of leaves have nothing to move: in neither list
      const bool single = d.start <= p && d.end >= p + kChunkW;
      if (!single || d.split) list_chunk(a.ctl->pcnt, a.plist, P, c, single);
    } else {
      const int64_t c = t - G - P;
      const int64_t p = c * kChunkW;
      const int f = (int)(p / (int64_t)A2);
      const int64_t fbase = (int64_t)f * (int64_t)A2;
      const uint32_t q = (uint32_t)(p - fbase);
      const uint32_t k = cache ? find_start(s2, K2, q) : find_node(a.next, K2, q);
      const NodeL nd = a.next[k];
      ChunkDesc d;
      d.start = fbase + nd.start;
      d.end = d.start + nd.N;
      d.k = k;
      d.f = f;
      d.c = nd.c;
      d.sc = nd.sc;
      d.v = nd.v;
      d.N = nd.N;
      d.srch = nd.searchable;
      a.sdesc[c] = d;
      list_chunk(a.ctl->scnt, a.slist, S, c, d.start <= p && d.end >= p + kChunkW);
    }
  }
}

struct PartArgs {
  const float* lx;
  const uint32_t* lr;
  const double* ly;
  float* ox;
  uint32_t* orow;
  double* oy;
  const NodeL* nodes;
  const Decision* dec;
  const uint32_t* new_start;
  const uint32_t* gbits;  // go-left bitmap (global)
  uint32_t* gmask;        // [nchunks * kRows] go-left ballots per row of 32 entries (phase A -> C)
  int64_t nwords;         // bitmap words
  const PartDesc* desc;  // per warp chunk
  const uint32_t* list;   // chunk list (prep_kernel): split singles first, others from the back
  const Ctl* ctl;
  int parity;
  int dl_in;   // lists in the input (d)
  int dl_out;  // lists to write (d, or 1 before the last level)
  CntP* chunk_agg;    // [nchunks] phase A
  CntP* chunk_excl;   // [nchunks] phase B1
  CntP* block_agg;
  CntP* block_carry;
};

// Stable partition of each (node, feature) segment: left rows first then right rows,
// order preserved; rows of nodes that did not split are dropped.
//
// Warp chunks of kChunkW = kRows x 32 consecutive entries (row r of a chunk = 32
// consecutive entries, lane = position in the row).  Within a row the left/right rank of
// every entry comes from two ballots (go-left mask, segment-head mask), so each child's
// entries of a row go to consecutive addresses (coalesced stores).  Carries: row to row
// inside the warp; chunk to chunk from phase A (per-chunk left counts) + the fixed-shape
// chunk scan (phase B, shared with the split scan).  No block barriers, no look-back.
constexpr int kRows = kChunkW / 32;  // rows of 32 per warp chunk

// Per-row head / split masks of a lane's kRows entries (cursor s advanced); gbits = the
// raw go-left bits masked by "node split".
__device__ __forceinline__ void part_flags(const PartArgs& a, uint32_t K, uint64_t A, int64_t wbase,
                                           int64_t total, Seg& s, uint32_t graw, uint32_t& gbits,
                                           uint32_t& hbits, uint32_t& sbits, const PartDesc& dsc) {
  const int lane = threadIdx.x & 31;
  hbits = sbits = 0;
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    const int64_t p = wbase + r * 32 + lane;
    if (p < total) {
      while (p >= s.end) seg_next(s, a.nodes, K, A);
      if (p == s.start) hbits |= 1u << r;
      const bool sp = (s.k == dsc.k && s.f == dsc.f) ? (dsc.split != 0) : (__ldg(&a.dec[s.k].f) >= 0);
      if (sp) sbits |= 1u << r;
    }
  }
  gbits = graw & sbits;
}

__device__ __forceinline__ void load_rows(const uint32_t* __restrict__ lr, int64_t wbase, int64_t total, uint32_t* rv) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    const int64_t p = wbase + r * 32 + lane;
    rv[r] = (p < total) ? __ldcs(lr + p) : 0u;
  }
}

// Largest go-left bitmap kept in shared memory by part_agg_kernel<true> (rows <= 1.8M).
constexpr int64_t kMaxSmemBitmapBytes = 227 * 1024;
constexpr int kAggSmemThreads = 1024;

// Phase A: per-chunk aggregate of go-left counts (lefts since the chunk's last head), and
// the chunk's raw go-left ballots (one word per row of 32 entries) for phase C, so the
// partition itself gathers nothing.  kSmem: the whole bitmap is staged in shared memory
// (one CTA per SM), so the per-entry gathers are shared-memory loads, not L2 round trips.
template <bool kSmem>
__global__ void __launch_bounds__(kSmem ? kAggSmemThreads : kThreads) part_agg_kernel(PartArgs a) {
  extern __shared__ uint4 smem_bits4[];
  const uint32_t* __restrict__ bits = kSmem ? reinterpret_cast<const uint32_t*>(smem_bits4) : a.gbits;
  const uint32_t K = a.ctl->K[a.parity];
  const uint64_t A = a.ctl->A[a.parity];
  const uint64_t A2 = a.ctl->A[a.parity ^ 1];
  if (K == 0 || A2 == 0) return;
  const int64_t total = (int64_t)A * a.dl_out;
  const int64_t nch = (total + kChunkW - 1) / kChunkW;
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  uint32_t rn[kRows];
  if (gw < nch) load_rows(a.lr, gw * kChunkW, total, rn);
  if (kSmem) {
    const int64_t n4 = (a.nwords + 3) / 4;
    const uint4* g4 = reinterpret_cast<const uint4*>(a.gbits);
    for (int64_t i = threadIdx.x; i < n4; i += blockDim.x) smem_bits4[i] = __ldg(g4 + i);
    __syncthreads();
  }
  for (int64_t ch = gw; ch < nch; ch += nw) {
    const int64_t wbase = ch * kChunkW;
    uint32_t rv[kRows];
#pragma unroll
    for (int r = 0; r < kRows; ++r) rv[r] = rn[r];
    if (ch + nw < nch) load_rows(a.lr, (ch + nw) * kChunkW, total, rn);
    const PartDesc dsc = a.desc[ch];
    uint32_t graw = 0;
#pragma unroll
    for (int r = 0; r < kRows; ++r) graw |= ((bits[rv[r] >> 5] >> (rv[r] & 31)) & 1u) << r;
    uint32_t my_mask = 0;
    if (dsc.start <= wbase && dsc.end >= wbase + kChunkW) {
      // whole chunk in one segment (a head can only be its first entry)
      uint32_t c = 0;
#pragma unroll
      for (int r = 0; r < kRows; ++r) {
        const uint32_t gm = __ballot_sync(0xffffffffu, (graw >> r) & 1u);
        if (lane == r) my_mask = gm;
        c += __popc(gm);
      }
      if (lane == 0) a.chunk_agg[ch] = CntP{dsc.start == wbase ? 1u : 0u, dsc.split ? c : 0u};
    } else {
      Seg s{0, 0, 0, 0u, 0};
      seg_from(s, dsc.start, dsc.end, dsc.k, dsc.f, A, min(wbase + lane, total - 1), a.nodes, K);
      uint32_t gbits, hbits, sbits;
      part_flags(a, K, A, wbase, total, s, graw, gbits, hbits, sbits, dsc);
      CntP agg{0u, 0u};
#pragma unroll
      for (int r = 0; r < kRows; ++r) {
        const uint32_t rm = __ballot_sync(0xffffffffu, (graw >> r) & 1u);
        if (lane == r) my_mask = rm;
        const uint32_t gm = __ballot_sync(0xffffffffu, (gbits >> r) & 1u);
        const uint32_t hm = __ballot_sync(0xffffffffu, (hbits >> r) & 1u);
        if (hm) {
          const int hl = 31 - __clz(hm);
          agg.flag = 1u;
          agg.c = __popc(gm & ~((1u << hl) - 1u));
        } else {
          agg.c += __popc(gm);
        }
      }
      if (lane == 0) a.chunk_agg[ch] = agg;
    }
    if (lane < kRows) a.gmask[ch * kRows + lane] = my_mask;
  }
}

// Phase C, one chunk inside ONE segment of a split node: ranks from the chunk's go-left
// ballots plus one carry; each child's entries of a row go to consecutive addresses.
// y moves as raw bits: 4 B (y32) or 8 B per entry.
__device__ __forceinline__ unsigned long long yload_raw(const double* __restrict__ ly, int64_t p, bool y32) {
  return y32 ? (unsigned long long)__ldcs(reinterpret_cast<const unsigned int*>(ly) + p)
             : (unsigned long long)__ldcs(reinterpret_cast<const unsigned long long*>(ly) + p);
}
__device__ __forceinline__ void ystore_raw(double* __restrict__ oy, int64_t o, unsigned long long v, bool y32) {
  if (y32) reinterpret_cast<unsigned int*>(oy)[o] = (unsigned int)v;
  else reinterpret_cast<unsigned long long*>(oy)[o] = v;
}

__device__ __forceinline__ void partition_single_chunk(const PartArgs& a, uint64_t A2, int64_t ch, bool y32) {
  const int lane = threadIdx.x & 31;
  const uint32_t lt_mask = (1u << lane) - 1u;
  const int64_t wbase = ch * kChunkW;
  uint32_t rv[kRows];
  float xv[kRows];
  unsigned long long yv[kRows];
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    const int64_t p = wbase + r * 32 + lane;
    rv[r] = __ldcs(a.lr + p);
    xv[r] = __ldcs(a.lx + p);
    yv[r] = yload_raw(a.ly, p, y32);
  }
  const PartDesc dsc = a.desc[ch];
  const uint32_t mword = (lane < kRows) ? __ldcs(a.gmask + ch * kRows + lane) : 0u;
  uint32_t carry = (dsc.start == wbase) ? 0u : combine(a.block_carry[ch / kBlockChunks], a.chunk_excl[ch]).c;
  const uint32_t i0 = (uint32_t)(wbase - dsc.start) + lane;
  const uint32_t nsl = dsc.ns + dsc.nl;
  float* const ox = a.ox + (int64_t)dsc.f * (int64_t)A2;
  uint32_t* const orow = a.orow + (int64_t)dsc.f * (int64_t)A2;
  const int64_t ybase = (int64_t)dsc.f * (int64_t)A2;
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    const uint32_t gm = __shfl_sync(0xffffffffu, mword, r);
    const uint32_t g = (gm >> lane) & 1u;
    const uint32_t rank = carry + __popc(gm & lt_mask);
    const uint32_t i = i0 + r * 32;
    const uint32_t dst = g ? dsc.ns + rank : nsl + (i - rank);
    ox[dst] = xv[r];
    orow[dst] = rv[r];
    ystore_raw(a.oy, ybase + dst, yv[r], y32);
    carry += __popc(gm);
  }
}

// Phase C, one chunk with segment boundaries inside.
__device__ __forceinline__ void partition_general_chunk(const PartArgs& a, uint32_t K, uint64_t A, uint64_t A2,
                                                      int64_t total, int64_t ch, bool y32) {
  const int lane = threadIdx.x & 31;
  const uint32_t lt_mask = (1u << lane) - 1u;
  const int64_t wbase = ch * kChunkW;
  uint32_t rv[kRows];
  float xv[kRows];
  unsigned long long yv[kRows];
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    const int64_t p = wbase + r * 32 + lane;
    const bool ok = p < total;
    rv[r] = ok ? __ldcs(a.lr + p) : 0u;
    xv[r] = ok ? __ldcs(a.lx + p) : 0.f;
    yv[r] = ok ? yload_raw(a.ly, p, y32) : 0ull;
  }
  const PartDesc dsc = a.desc[ch];
  // raw go-left bits of my kRows entries, from the chunk's ballots (phase A)
  const uint32_t mword = (lane < kRows) ? __ldcs(a.gmask + ch * kRows + lane) : 0u;
  uint32_t graw = 0;
#pragma unroll
  for (int r = 0; r < kRows; ++r) graw |= ((__shfl_sync(0xffffffffu, mword, r) >> lane) & 1u) << r;
  Seg s{0, 0, 0, 0u, 0};
  seg_from(s, dsc.start, dsc.end, dsc.k, dsc.f, A, min(wbase + lane, total - 1), a.nodes, K);
  const Seg s0 = s;
  uint32_t gbits, hbits, sbits;
  part_flags(a, K, A, wbase, total, s, graw, gbits, hbits, sbits, dsc);
  const CntP cc = combine(a.block_carry[ch / kBlockChunks], a.chunk_excl[ch]);
  uint32_t carry = cc.c;  // lefts of the open segment before this chunk
  s = s0;
  uint32_t nlv = 0, nsv = 0;
  int64_t obase = 0;
  uint32_t cur_k = 0xffffffffu;
  int cur_f = -1;
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    const int64_t p = wbase + r * 32 + lane;
    const uint32_t g = (gbits >> r) & 1u, sp = (sbits >> r) & 1u;
    const uint32_t gm = __ballot_sync(0xffffffffu, g);
    const uint32_t hm = __ballot_sync(0xffffffffu, (hbits >> r) & 1u);
    if (p < total) {
      while (p >= s.end) seg_next(s, a.nodes, K, A);
      if (sp) {
        if (s.k != cur_k || s.f != cur_f) {
          cur_k = s.k;
          cur_f = s.f;
          const bool ind = (s.k == dsc.k && s.f == dsc.f);
          nlv = ind ? dsc.nl : __ldg(&a.dec[s.k].nl);
          nsv = ind ? dsc.ns : __ldg(&a.new_start[s.k]);
          obase = (int64_t)s.f * (int64_t)A2;
        }
        const uint32_t le = hm & ((lt_mask << 1) | 1u);  // heads at lanes <= me
        uint32_t rank;
        if (le) {
          const int hl = 31 - __clz(le);
          rank = __popc(gm & lt_mask & ~((1u << hl) - 1u));
        } else {
          rank = carry + __popc(gm & lt_mask);
        }
        const uint32_t i = (uint32_t)(p - s.start);
        const uint32_t dst = g ? nsv + rank : nsv + nlv + (i - rank);
        const int64_t o = obase + dst;
        a.ox[o] = xv[r];
        a.orow[o] = rv[r];
        ystore_raw(a.oy, o, yv[r], y32);
      }
    }
    if (hm) {
      const int hl = 31 - __clz(hm);
      carry = __popc(gm & ~((1u << hl) - 1u));
    } else {
      carry += __popc(gm);
    }
  }
}

// Phase C: the level's chunk list, single-segment chunks of split nodes first, then the
// chunks with segment boundaries (chunks of leaves inside one segment are not listed).
#ifndef DT_PART_MINB
#define DT_PART_MINB 3  // 3 CTAs/SM: no register spills (measured: 4 -> 3 saves ~2% of the partition)
#endif
__global__ void __launch_bounds__(kThreads, DT_PART_MINB) partition_kernel(PartArgs a) {
  const uint32_t K = a.ctl->K[a.parity];
  const uint64_t A = a.ctl->A[a.parity];
  const uint64_t A2 = a.ctl->A[a.parity ^ 1];
  if (K == 0 || A2 == 0) return;
  const int64_t total = (int64_t)A * a.dl_out;  // only the lists we write
  const int64_t nch = (total + kChunkW - 1) / kChunkW;
  const int64_t ns = a.ctl->pcnt[0], ng = a.ctl->pcnt[1];
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const bool y32 = a.ctl->y32 != 0;
  for (int64_t idx = gw; idx < ns + ng; idx += nw) {
    if (idx < ns) partition_single_chunk(a, A2, (int64_t)a.list[idx], y32);
    else partition_general_chunk(a, K, A, A2, total, (int64_t)a.list[nch - 1 - (idx - ns)], y32);
  }
}

// ----------------------------------------------------------------------------- driver --

template <class T>
cudaError_t dmalloc(T** p, size_t count, cudaStream_t s) {
  return cudaMallocAsync((void**)p, sizeof(T) * (count ? count : 1), s);
}

struct Workspace {
  std::vector<void*> ptrs;
  cudaStream_t s;
  ~Workspace() {
    for (void* p : ptrs) cudaFreeAsync(p, s);
  }
  template <class T>
  cudaError_t get(T** p, size_t count) {
    cudaError_t e = dmalloc(p, count, s);
    if (e == cudaSuccess) ptrs.push_back(*p);
    return e;
  }
};

int persistent_grid(const void* kern, int threads, size_t smem) {
  int per = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, kern, threads, smem);
  if (per < 1) per = 1;
  return num_sms() * per;
}

// ----------------------------------------------------------------------------- buffers --

struct FitBufs {
  float* lx[2];
  uint32_t* lr[2];
  double* ly[2];
  NodeL* nodes[2];
  Decision* dec;
  uint32_t* new_start;
  Cand *head_cand, *cont_cand;
  unsigned long long* slot_gain;
  uint32_t* slot_pos;
  Stat *head_stat, *cont_stat;
  uint32_t* gbits;  // go-left bitmap, nwords4 words
  uint32_t* gmask;  // [max_chunks * kRows]
  int64_t nwords4;
  dt_node* dout;
  Ctl* ctl;
  LevelLog* lvlog;
  RootPart* parts;
  double* cparts;
  uint32_t *k_in, *k_out;  // per feature: n keys flip(x), stable-sorted feature by feature
  uint32_t *v_in, *v_out;
  uint32_t *rs_cnt, *rs_off;  // batched tile sort: per (feature, digit, tile) counts / offsets
  uint32_t* rs_tot;           // per (feature, digit) totals
  int rs_tiles;               // radix-sort tiles per feature
  ChunkDesc* sdesc;
  uint32_t *slist, *plist;  // per-level chunk lists (scan, partition)
  PartDesc* pdesc;
  SumP *chunk_agg, *chunk_excl, *block_agg, *block_carry;
  CntP *pchunk_agg, *pchunk_excl, *pblock_agg, *pblock_carry;
  ExchRec *exch_send, *exch_all;
  int64_t kcap, out_cap, max_chunks, max_cblocks, root_np, root_chunk;
  int fbits;
};

// Feature sharding context: this rank owns global features j * world + rank.
struct ShardCtx {
  dt_comm* comm;
  int world, rank, dg;
};

// Allocates every buffer through `get` (stream-ordered or persistent).
template <class Get>
dt_status fit_alloc(FitBufs& b, int64_t n, int32_t d, int32_t max_depth, int world, Get get) {
  const int64_t total0 = n * (int64_t)d;
  b.kcap = n;
  if (max_depth >= 0 && max_depth < 40) b.kcap = std::min<int64_t>(b.kcap, (int64_t)1 << max_depth);
  b.out_cap = 2 * n - 1;
  if (max_depth >= 0 && max_depth < 40) b.out_cap = std::min<int64_t>(b.out_cap, ((int64_t)1 << (max_depth + 1)) - 1);
  if (b.out_cap >= ((int64_t)1 << 31)) return fail(DT_ERR_TOO_LARGE, "dt_fit: node array too large");
  b.max_chunks = (total0 + kChunkW - 1) / kChunkW + 1;
  b.max_cblocks = (b.max_chunks + kBlockChunks - 1) / kBlockChunks + 1;
  b.root_chunk = 8192;
  b.root_np = (n + b.root_chunk - 1) / b.root_chunk;
  if (b.root_np > 2048) {
    b.root_np = 2048;
    b.root_chunk = (n + b.root_np - 1) / b.root_np;
    b.root_np = (n + b.root_chunk - 1) / b.root_chunk;
  }
  b.fbits = 0;
  while ((1 << b.fbits) < d) ++b.fbits;
  if (b.fbits > 8) b.fbits = 8;
  for (int k = 0; k < 2; ++k) {
    DT_CK(get(&b.lx[k], (size_t)total0));
    DT_CK(get(&b.lr[k], (size_t)total0));
    DT_CK(get(&b.ly[k], (size_t)total0));
    DT_CK(get(&b.nodes[k], (size_t)b.kcap + 1));
  }
  DT_CK(get(&b.dec, (size_t)b.kcap));
  DT_CK(get(&b.new_start, (size_t)b.kcap));
  DT_CK(get(&b.head_cand, (size_t)b.kcap * d));
  DT_CK(get(&b.slot_gain, (size_t)b.kcap * d));
  DT_CK(get(&b.slot_pos, (size_t)b.kcap * d));
  DT_CK(get(&b.cont_cand, (size_t)b.max_chunks));
  DT_CK(get(&b.head_stat, (size_t)b.kcap));
  DT_CK(get(&b.cont_stat, (size_t)b.max_chunks));
  b.nwords4 = ((n + 127) / 128) * 4;  // whole uint4s
  DT_CK(get(&b.gbits, (size_t)b.nwords4));
  DT_CK(get(&b.gmask, (size_t)b.max_chunks * kRows));
  DT_CK(get(&b.dout, (size_t)b.out_cap));
  DT_CK(get(&b.ctl, 1));
  DT_CK(get(&b.lvlog, (size_t)kMaxLogLevels));
  DT_CK(get(&b.parts, (size_t)b.root_np));
  DT_CK(get(&b.cparts, (size_t)b.root_np));
  // the presort's key / row buffers live in the level-1 lists (16 B per entry = exactly
  // the four 4-B arrays): they are dead once presort_build has written the level-0 lists,
  // before level 0's partition first writes lists[1].  Saves 16 B per entry (C3: 51 GB).
  b.k_in = reinterpret_cast<uint32_t*>(b.lx[1]);
  b.k_out = b.lr[1];
  b.v_in = reinterpret_cast<uint32_t*>(b.ly[1]);
  b.v_out = reinterpret_cast<uint32_t*>(b.ly[1]) + total0;
  b.rs_tiles = (int)((n + kTile - 1) / kTile);
  DT_CK(get(&b.rs_cnt, (size_t)d * 256 * b.rs_tiles));
  DT_CK(get(&b.rs_off, (size_t)d * 256 * b.rs_tiles));
  DT_CK(get(&b.rs_tot, (size_t)d * 256));
  DT_CK(get(&b.sdesc, (size_t)b.max_chunks));
  DT_CK(get(&b.slist, (size_t)b.max_chunks));
  DT_CK(get(&b.plist, (size_t)b.max_chunks));
  DT_CK(get(&b.pdesc, (size_t)b.max_chunks));
  DT_CK(get(&b.chunk_agg, (size_t)b.max_chunks));
  DT_CK(get(&b.chunk_excl, (size_t)b.max_chunks));
  DT_CK(get(&b.block_agg, (size_t)b.max_cblocks));
  DT_CK(get(&b.block_carry, (size_t)b.max_cblocks));
  DT_CK(get(&b.pchunk_agg, (size_t)b.max_chunks));
  DT_CK(get(&b.pchunk_excl, (size_t)b.max_chunks));
  DT_CK(get(&b.pblock_agg, (size_t)b.max_cblocks));
  DT_CK(get(&b.pblock_carry, (size_t)b.max_cblocks));
  DT_CK(get(&b.exch_send, (size_t)b.kcap));
  if (world > 1) DT_CK(get(&b.exch_all, (size_t)b.kcap * world));
  else b.exch_all = b.exch_send;
  return DT_OK;
}


// profiling records whose bytes depend on device-side counts
struct Pending {
  int rec, level, kind, dl;
};

// Enqueues the whole fit on stream s (no host synchronisation unless `poll`).
dt_status fit_enqueue(const FitBufs& b, const float* X, const double* y, int64_t n, int32_t d,
                      int32_t max_depth, int64_t min_leaf, cudaStream_t s, bool poll,
                      std::vector<Pending>* pending, const ShardCtx& sh) {
  const int64_t total0 = n * (int64_t)d;
  DT_CK(cudaMemsetAsync(b.slot_gain, 0, sizeof(unsigned long long) * (size_t)b.kcap * d, s));
  // piece records carry the level that wrote them; none may match before it is written
  DT_CK(cudaMemsetAsync(b.head_cand, 0xFF, sizeof(Cand) * (size_t)b.kcap * d, s));
  DT_CK(cudaMemsetAsync(b.slot_pos, 0xFF, sizeof(uint32_t) * (size_t)b.kcap * d, s));
  DT_CK(cudaMemsetAsync(b.cont_cand, 0xFF, sizeof(Cand) * (size_t)b.max_chunks, s));
  DT_CK(cudaMemsetAsync(b.ctl, 0, sizeof(Ctl), s));
  Ctl* ctl = b.ctl;
  // ---- root statistics (a0: N, sum y, min/max, integrality, finiteness, centre)
  {
    const int pr = prof_begin(PK_ROOT, s, 4);
    root_reduce_kernel<<<(unsigned)b.root_np, 256, 0, s>>>(y, n, b.root_chunk, b.parts);
    root_finalize_kernel<<<1, 32, 0, s>>>(b.parts, (int)b.root_np, n, ctl);
    root_center_kernel<<<(unsigned)b.root_np, 256, 0, s>>>(y, n, b.root_chunk, ctl, b.cparts);
    root_init_kernel<<<1, 32, 0, s>>>(b.cparts, (int)b.root_np, n, max_depth, min_leaf, ctl, b.nodes[0]);
    prof_end(pr, s, 16.0 * (double)n);  // y read twice
    DT_CK(cudaGetLastError());
  }
  // ---- presort (a2): per-feature stable sort of (x, row), SoA level-0 lists
  {
    const int rb = sh.dg <= 48 ? 256 : (sh.dg <= 96 ? 128 : 64);  // rows per block (smem)
    const int64_t nb = (n + rb - 1) / rb;
    const size_t smem = sizeof(float) * rb * (size_t)sh.dg;
    if (smem > 48 * 1024)
      DT_CK(cudaFuncSetAttribute(presort_keys_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int pr = prof_begin(PK_PRESORT_KEYS, s, 1);
    presort_keys_kernel<<<(unsigned)nb, 256, smem, s>>>(X, n, d, b.k_in, b.v_in, ctl, sh.dg, sh.world,
                                                        sh.rank, rb);
    prof_end(pr, s, 16.0 * (double)total0);  // X read + (key, val) written
    DT_CK(cudaGetLastError());
    // stable 32-bit radix sort of every feature's n keys (4 passes each; ties keep the
    // row order -> (x, row id) order), the d sorts forked over side streams
    const uint32_t* sk = b.k_out;  // sorted keys / rows
    const uint32_t* sv = b.v_out;
    {
      // batched tile radix sort of all d lists: 4 passes x 3 launches (ping-pong, ends in _in)
      pr = prof_begin(PK_PRESORT_SORT, s, 12);
      uint32_t *ki = b.k_in, *ko = b.k_out, *vi = b.v_in, *vo = b.v_out;
      const dim3 g((unsigned)b.rs_tiles, (unsigned)d);
      for (int pass = 0; pass < 4; ++pass) {
        const int shift = 8 * pass;
        rs_count_kernel<<<g, kTS, 0, s>>>(ki, n, shift, b.rs_tiles, b.rs_cnt);
        rs_offset_kernel<<<dim3(256, (unsigned)d), std::min(1024, (b.rs_tiles + 31) / 32 * 32), 0, s>>>(
            b.rs_cnt, b.rs_tiles, b.rs_off, b.rs_tot);
        rs_scatter_kernel<<<g, kTS, 0, s>>>(ki, vi, ko, vo, n, shift, b.rs_tiles, b.rs_off, b.rs_tot);
        std::swap(ki, ko);
        std::swap(vi, vo);
      }
      prof_end(pr, s, 4.0 * 24.0 * (double)total0);  // per pass: keys read twice, pairs read + written
      DT_CK(cudaGetLastError());
      sk = ki;
      sv = vi;
    }
    const int gb = std::max(1, std::min<int>((int)((total0 + 255) / 256), num_sms() * 8));
    pr = prof_begin(PK_PRESORT_BUILD, s, 1);
    presort_build_kernel<<<gb, 256, 0, s>>>(sk, sv, y, total0, b.lx[0], b.lr[0], b.ly[0], ctl);
    prof_end(pr, s, 36.0 * (double)total0);  // (key, val) read, y gathered, 16 B written
    DT_CK(cudaGetLastError());
  }
  const int g_scan = persistent_grid((const void*)scan_kernel, kThreads, 0);
  DT_CK(cudaFuncSetAttribute((const void*)scan_single_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)kScanSingleSmem));
  const int g_scan1 = persistent_grid((const void*)scan_single_kernel, kThreads, kScanSingleSmem);
  DT_CK(cudaFuncSetAttribute((const void*)scan_agg_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)kScanAggSmem));
  const int g_agg = persistent_grid((const void*)scan_agg_kernel, kThreads, kScanAggSmem);
  const int g_pagg = persistent_grid((const void*)part_agg_kernel<false>, kThreads, 0);
  size_t agg_smem = sizeof(uint32_t) * (size_t)b.nwords4;
  if ((int64_t)agg_smem > kMaxSmemBitmapBytes) agg_smem = 0;
  else DT_CK(cudaFuncSetAttribute((const void*)part_agg_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  (int)agg_smem));
  const int g_part = persistent_grid((const void*)partition_kernel, kThreads, 0);
  const int g_sel = num_sms() * 4;
  const int g_gl = num_sms() * 8;

  int cur = 0;
  for (int level = 0;; ++level) {
    const int parity = level & 1;
    const bool last = (max_depth >= 0 && level == max_depth);
    const int dl = last ? 1 : d;
    // scan (a4)
    int pr = prof_begin(PK_SCAN, s, level == 0 ? 5 : 4);
    // level 0's chunk descriptors; deeper levels' come from the previous level's prep_kernel
    if (level == 0) scan_desc_kernel<<<num_sms() * 4, 256, 0, s>>>(b.nodes[parity], ctl, parity, dl, kChunkW, b.sdesc, b.slist);
    ScanArgs sa;
    sa.desc = b.sdesc;
    sa.list = b.slist;
    sa.lx = b.lx[cur];
    sa.ly = b.ly[cur];
    sa.nodes = b.nodes[parity];
    sa.ctl = ctl;
    sa.parity = parity;
    sa.dl = dl;
    sa.d = d;
    sa.min_leaf = min_leaf;
    sa.chunk_agg = b.chunk_agg;
    sa.chunk_excl = b.chunk_excl;
    sa.block_agg = b.block_agg;
    sa.block_carry = b.block_carry;
    sa.head_cand = b.head_cand;
    sa.cont_cand = b.cont_cand;
    sa.head_stat = b.head_stat;
    sa.cont_stat = b.cont_stat;
    sa.slot_gain = b.slot_gain;
    sa.level = (uint32_t)level;
    scan_agg_kernel<<<g_agg, kThreads, kScanAggSmem, s>>>(sa);
    chunk_scan_kernel<SumP><<<(unsigned)b.max_cblocks, 1024, 0, s>>>(ctl, parity, dl, b.chunk_agg, b.chunk_excl,
                                                                     b.block_agg, b.block_carry);
    scan_single_kernel<<<g_scan1, kThreads, kScanSingleSmem, s>>>(sa);
    scan_kernel<<<g_scan, kThreads, 0, s>>>(sa);
    prof_end(pr, s, 0.0);
    if (pending) pending->push_back({pr, level, PK_SCAN, dl});
    DT_CK(cudaGetLastError());
    // select (a5, a8)
    SelectArgs se;
    se.lx = b.lx[cur];
    se.nodes = b.nodes[parity];
    se.ctl = ctl;
    se.parity = parity;
    se.level = level;
    se.dl = dl;
    se.d = d;
    se.head_cand = b.head_cand;
    se.cont_cand = b.cont_cand;
    se.head_stat = b.head_stat;
    se.cont_stat = b.cont_stat;
    se.dec = b.dec;
    se.out = b.dout;
    se.log = b.lvlog;
    se.slot_gain = b.slot_gain;
    se.slot_pos = b.slot_pos;
    se.exch = b.exch_send;
    se.gbits = reinterpret_cast<uint4*>(b.gbits);
    se.nvec = b.nwords4 / 4;
    se.world = sh.world;
    se.rank = sh.rank;
    se.dg = sh.dg;
    pr = prof_begin(PK_SELECT, s, sh.world > 1 ? 3 : 2);
    piece_pos_kernel<<<num_sms() * 4, 256, 0, s>>>(sa, b.slot_pos);
    select_kernel<<<g_sel, 256, 0, s>>>(se);
    // exchange the per-node local bests (at most min(kcap, 2^level) nodes at this level)
    const int64_t cnt = (level < 40) ? std::min<int64_t>(b.kcap, (int64_t)1 << level) : b.kcap;
    if (sh.world > 1) {
      dt_status cst = comm_allgather(sh.comm, b.exch_send, b.exch_all, sizeof(ExchRec) * (size_t)cnt, s);
      if (cst != DT_OK) return cst;
    }
    if (sh.world > 1)  // (a single rank decides inside select_kernel)
      decide_kernel<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>((cnt + 255) / 256, num_sms() * 4)), 256, 0, s>>>(
          se, b.exch_all, cnt);
    prof_end(pr, s, 0.0);
    DT_CK(cudaGetLastError());
    if (last) break;
    // number (a3, a8)
    NumberArgs na;
    na.nodes = b.nodes[parity];
    na.next = b.nodes[parity ^ 1];
    na.dec = b.dec;
    na.new_start = b.new_start;
    na.ctl = ctl;
    na.parity = parity;
    na.level = level;
    na.max_depth = max_depth;
    na.min_leaf = min_leaf;
    na.out = b.dout;
    na.log = b.lvlog;
    pr = prof_begin(PK_NUMBER, s, 1);
    number_kernel<<<1, 1024, 0, s>>>(na);
    prof_end(pr, s, 0.0);
    DT_CK(cudaGetLastError());
    // go-left map (a6) + this level's partition descriptors + the next level's scan
    // descriptors (one launch)
    const int dl_out = (max_depth >= 0 && level + 1 == max_depth) ? 1 : d;
    pr = prof_begin(PK_GOLEFT, s, 1);
    {
      PrepArgs pp;
      pp.lr = b.lr[cur];
      pp.nodes = b.nodes[parity];
      pp.next = b.nodes[parity ^ 1];
      pp.dec = b.dec;
      pp.new_start = b.new_start;
      pp.gbits = b.gbits;
      pp.pdesc = b.pdesc;
      pp.plist = b.plist;
      pp.sdesc = b.sdesc;
      pp.slist = b.slist;
      pp.ctl = ctl;
      pp.parity = parity;
      pp.dl_out = dl_out;
      prep_kernel<<<num_sms() * (1024 / kPrepThreads), kPrepThreads, 0, s>>>(pp);
    }
    if (sh.world > 1) {
      // only the owner of each split feature set its rows' bits: OR over the ranks
      dt_status cst = comm_allreduce_or_u32(sh.comm, b.gbits, b.nwords4, s);
      if (cst != DT_OK) return cst;
    }
    prof_end(pr, s, 0.0);
    if (pending) pending->push_back({pr, level, PK_GOLEFT, 1});
    DT_CK(cudaGetLastError());
    // stable partition (a7)
    PartArgs pa;
    pa.lx = b.lx[cur];
    pa.lr = b.lr[cur];
    pa.ly = b.ly[cur];
    pa.ox = b.lx[cur ^ 1];
    pa.orow = b.lr[cur ^ 1];
    pa.oy = b.ly[cur ^ 1];
    pa.nodes = b.nodes[parity];
    pa.dec = b.dec;
    pa.new_start = b.new_start;
    pa.gbits = b.gbits;
    pa.gmask = b.gmask;
    pa.nwords = b.nwords4;
    pa.desc = b.pdesc;
    pa.ctl = ctl;
    pa.parity = parity;
    pa.dl_in = d;
    pa.dl_out = dl_out;
    pa.chunk_agg = b.pchunk_agg;
    pa.chunk_excl = b.pchunk_excl;
    pa.block_agg = b.pblock_agg;
    pa.block_carry = b.pblock_carry;
    pr = prof_begin(PK_PARTITION, s, 3);
    pa.list = b.plist;
    if (agg_smem) part_agg_kernel<true><<<num_sms(), kAggSmemThreads, agg_smem, s>>>(pa);
    else part_agg_kernel<false><<<g_pagg, kThreads, 0, s>>>(pa);
    chunk_scan_kernel<CntP><<<(unsigned)b.max_cblocks, 1024, 0, s>>>(ctl, parity, pa.dl_out, b.pchunk_agg,
                                                                     b.pchunk_excl, b.pblock_agg, b.pblock_carry);
    partition_kernel<<<g_part, kThreads, 0, s>>>(pa);
    prof_end(pr, s, 0.0);
    if (pending) pending->push_back({pr, level, PK_PARTITION, pa.dl_out});
    DT_CK(cudaGetLastError());
    cur ^= 1;
    // unlimited depth (or a deep limit): poll the node count every few levels
    if (poll && (max_depth < 0 || max_depth > 24) && (level % 8) == 7) {
      uint32_t kk[2];
      DT_CK(cudaMemcpyAsync(kk, ctl->K, sizeof kk, cudaMemcpyDeviceToHost, s));
      DT_CK(cudaStreamSynchronize(s));
      if (kk[parity ^ 1] == 0) break;
    }
  }
  return DT_OK;
}

// Device-side packing of the predict representation (see tree_upload in api.cu): the
// 8-byte packed form, or the 16-byte wide form for trees of >= kWideNodes nodes.
__global__ void __launch_bounds__(256) pack_tree_kernel(const dt_node* __restrict__ nodes, int64_t count,
                                                        uint2* __restrict__ packed, uint4* __restrict__ wide,
                                                        double* __restrict__ value) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < count; k += (int64_t)gridDim.x * blockDim.x) {
    const dt_node nd = nodes[k];
    value[k] = nd.value;
    uint32_t bits, left, feat;
    if (nd.feature < 0) {
      bits = 0x7f800000u;  // +inf, self-loop
      left = (uint32_t)k;
      feat = 0u;
    } else {
      bits = __float_as_uint(__double2float_rd(nd.threshold));  // x <= t  <=>  x <= RD32(t)
      left = (uint32_t)nd.left;
      feat = (uint32_t)nd.feature;
    }
    if (wide) wide[k] = make_uint4(bits, left, feat, 0u);
    else packed[k] = make_uint2(bits, (feat << 24) | left);
  }
}

// Reads the result back and builds the tree object (host nodes + device packed copy).
dt_status fit_finish(const FitBufs& b, int32_t d, cudaStream_t s, const std::vector<Pending>* pending,
                     dt_tree** out) {  // d = global feature count
  Ctl hc;
  DT_CK(cudaMemcpyAsync(&hc, b.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
  std::vector<LevelLog> hlog;
  if (pending && !pending->empty()) {
    hlog.resize(kMaxLogLevels);
    DT_CK(cudaMemcpyAsync(hlog.data(), b.lvlog, sizeof(LevelLog) * kMaxLogLevels, cudaMemcpyDeviceToHost, s));
  }
  DT_CK(cudaStreamSynchronize(s));
  if (pending) {
    // algorithmic bytes per launch:
    //   scan: every active entry of the scanned lists, x (4 B) + y (8 B, or 4 B as int32);
    //   goleft: the split feature's row ids of the moved rows (4 B, left rows only read, counted
    //           for all) + one bit per row;
    //   partition: every moved entry read and written (x 4 + row 4 + y 8 or 4 B, each way).
    for (const Pending& p : *pending) {
      if (p.rec < 0 || p.level >= kMaxLogLevels) continue;
      const LevelLog& L = hlog[(size_t)p.level];
      double bytes = 0.0;
      const double yb = hc.y32 ? 4.0 : 8.0;  // y bytes per entry (Reading R24)
      if (p.kind == PK_SCAN) bytes = (4.0 + yb) * (double)L.A * p.dl;
      else if (p.kind == PK_GOLEFT) bytes = 4.125 * (double)L.A_next;
      else if (p.kind == PK_PARTITION) bytes = 2.0 * (8.0 + yb) * (double)L.A_next * p.dl;
      prof_set_bytes(p.rec, bytes);
    }
  }
  if (hc.nonfinite) return fail(DT_ERR_NONFINITE, "dt_fit: non-finite value in X or y");
  const int64_t count = hc.next_id;
  dt_tree* t = new dt_tree();
  t->count = count;
  t->d = d;
  t->depth = hc.max_depth_seen;
  t->split_evals = (int64_t)hc.split_evals;
  t->integer_mode = hc.int_mode;
  t->host = (dt_node*)malloc(sizeof(dt_node) * (size_t)count);
  DT_CK(cudaGetDevice(&t->device));
  const bool wide = count >= kWideNodes;
  cudaError_t e = wide ? cudaMalloc((void**)&t->dev_wide, sizeof(uint4) * (size_t)count)
                       : cudaMalloc((void**)&t->dev_packed, sizeof(uint2) * (size_t)count);
  if (e == cudaSuccess) e = cudaMalloc((void**)&t->dev_value, sizeof(double) * (size_t)count);
  if (e == cudaSuccess) {
    const int g = (int)std::min<int64_t>((count + 255) / 256, 1024);
    pack_tree_kernel<<<g, 256, 0, s>>>(b.dout, count, t->dev_packed, t->dev_wide, t->dev_value);
    prof_add_launches(1);
    e = cudaGetLastError();
  }
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(t->host, b.dout, sizeof(dt_node) * (size_t)count, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) {
    dt_tree_free(t);
    return cuda_fail(e, "fit readback", __FILE__, __LINE__);
  }
  *out = t;
  return DT_OK;
}

// One cached, instantiated CUDA graph of a whole bounded-depth fit: replayed when the
// same inputs (addresses) and shape are fitted again (no per-launch host overhead).
struct FitPlan {
  const float* X = nullptr;
  const double* y = nullptr;
  int64_t n = 0, min_leaf = 0;
  int32_t d = 0, max_depth = 0;
  int device = -1;
  std::vector<void*> mem;
  FitBufs b{};
  cudaGraphExec_t exec = nullptr;
  cudaStream_t cap = nullptr;
  int64_t launches = 0;
  uint64_t last_use = 0;
  ~FitPlan() {
    if (exec) cudaGraphExecDestroy(exec);
    if (cap) cudaStreamDestroy(cap);
    for (void* p : mem) cudaFree(p);
  }
};
// Two cached plans (least recently used replaced): a caller alternating between two
// input buffers -- e.g. double-buffered host->device copies overlapping the previous fit
// -- replays both graphs without re-capture.  A plan whose workspace does not fit beside
// the other evicts it.
constexpr int kPlans = 2;
std::mutex g_plan_mu;
std::unique_ptr<FitPlan> g_plans[kPlans];
uint64_t g_plan_tick = 0;

}  // namespace

dt_status release_workspace_impl() {
  {
    std::lock_guard<std::mutex> lk(g_plan_mu);
    for (auto& p : g_plans) p.reset();
  }
  forest_release_scratch();
  DT_CK(cudaDeviceSynchronize());
  int dev = 0;
  DT_CK(cudaGetDevice(&dev));
  cudaMemPool_t pool;
  DT_CK(cudaDeviceGetDefaultMemPool(&pool, dev));
  DT_CK(cudaMemPoolTrimTo(pool, 0));
  return DT_OK;
}

dt_status fit_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t max_depth,
                   int64_t min_leaf, cudaStream_t s, dt_tree** out) {
  // Pool: keep freed workspace for the next fit (no cudaMalloc on the hot path).
  int dev = 0;
  DT_CK(cudaGetDevice(&dev));
  {
    cudaMemPool_t pool;
    DT_CK(cudaDeviceGetDefaultMemPool(&pool, dev));
    uint64_t thr = UINT64_MAX;
    DT_CK(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
  }
  static int graph_env = -1;
  if (graph_env < 0) {
    const char* e = getenv("DT_FIT_GRAPH");
    graph_env = (e && e[0] == '0') ? 0 : 1;
  }
  const bool use_graph = graph_env && !prof_enabled() && max_depth >= 0 && max_depth <= 24;
  if (use_graph) {
    std::lock_guard<std::mutex> lk(g_plan_mu);
    FitPlan* pl = nullptr;
    for (auto& p : g_plans)
      if (p && p->X == X && p->y == y && p->n == n && p->d == d && p->max_depth == max_depth &&
          p->min_leaf == min_leaf && p->device == dev)
        pl = p.get();
    if (!pl) {
      // victim slot: an empty one, else the least recently used
      int v = 0;
      for (int i = 0; i < kPlans; ++i) {
        if (!g_plans[i]) { v = i; break; }
        if (g_plans[i]->last_use < g_plans[v]->last_use) v = i;
      }
      FitPlan* old = g_plans[v].get();
      std::unique_ptr<FitPlan> np(new FitPlan());
      const bool same_shape = old && old->n == n && old->d == d && old->max_depth == max_depth && old->device == dev;
      if (same_shape) {
        // same buffer shapes (e.g. a min_samples_leaf grid, or new input addresses): keep
        // the workspace, re-capture only -- no cudaFree / cudaMalloc of ~32 B per entry
        DT_CK(cudaDeviceSynchronize());  // the old graph may still run on another stream
        np->mem.swap(old->mem);
        np->b = old->b;
        np->cap = old->cap;
        old->cap = nullptr;
      }
      g_plans[v].reset();  // frees the victim's memory unless it was taken over (synchronising)
      np->X = X;
      np->y = y;
      np->n = n;
      np->d = d;
      np->max_depth = max_depth;
      np->min_leaf = min_leaf;
      np->device = dev;
      if (!same_shape) {
        auto get = [&](auto** p, size_t count) -> cudaError_t {
          cudaError_t e = cudaMalloc((void**)p, sizeof(**p) * (count ? count : 1));
          if (e == cudaSuccess) np->mem.push_back((void*)*p);
          return e;
        };
        dt_status st = fit_alloc(np->b, n, d, max_depth, 1, get);
        if (st != DT_OK) {
          // no room beside the other cached plan(s): drop them and try once more
          bool others = false;
          for (auto& p : g_plans) others |= (bool)p;
          if (!others) return st;
          (void)cudaGetLastError();  // the failed cudaMalloc (not sticky)
          for (void* m : np->mem) cudaFree(m);
          np->mem.clear();
          np->b = FitBufs{};
          for (auto& p : g_plans) p.reset();
          st = fit_alloc(np->b, n, d, max_depth, 1, get);
          if (st != DT_OK) return st;
        }
        DT_CK(cudaStreamCreateWithFlags(&np->cap, cudaStreamNonBlocking));
      }
      const int64_t l0 = dt_launch_count();
      DT_CK(cudaStreamBeginCapture(np->cap, cudaStreamCaptureModeThreadLocal));
      dt_status st = fit_enqueue(np->b, X, y, n, d, max_depth, min_leaf, np->cap, false, nullptr,
                                 ShardCtx{nullptr, 1, 0, d});
      cudaGraph_t graph = nullptr;
      cudaError_t ce = cudaStreamEndCapture(np->cap, &graph);
      if (st != DT_OK) {
        if (graph) cudaGraphDestroy(graph);
        return st;
      }
      if (ce != cudaSuccess) return cuda_fail(ce, "cudaStreamEndCapture", __FILE__, __LINE__);
      np->launches = dt_launch_count() - l0;
      prof_add_launches(-np->launches);  // counted when replayed
      ce = cudaGraphInstantiate(&np->exec, graph, 0);
      cudaGraphDestroy(graph);
      if (ce != cudaSuccess) return cuda_fail(ce, "cudaGraphInstantiate", __FILE__, __LINE__);
      g_plans[v] = std::move(np);
      pl = g_plans[v].get();
    }
    pl->last_use = ++g_plan_tick;
    DT_CK(cudaGraphLaunch(pl->exec, s));
    prof_add_launches(pl->launches);
    return fit_finish(pl->b, d, s, nullptr, out);
  }
  // Direct path: stream-ordered workspace, kernels enqueued one by one.
  Workspace ws;
  ws.s = s;
  FitBufs b{};
  auto get = [&](auto** p, size_t count) -> cudaError_t { return ws.get(p, count); };
  dt_status st = fit_alloc(b, n, d, max_depth, 1, get);
  if (st != DT_OK) return st;
  std::vector<Pending> pending;
  st = fit_enqueue(b, X, y, n, d, max_depth, min_leaf, s, true, &pending, ShardCtx{nullptr, 1, 0, d});
  if (st != DT_OK) return st;
  return fit_finish(b, d, s, &pending, out);
}

// Feature-sharded fit: every rank holds the full table and builds /
// scans the feature lists j * world + rank; per level the ranks exchange their per-node
// best splits (allgather) and the go-left bitmap (OR-allreduce).  Same tree on every rank.
dt_status fit_sharded_impl(dt_comm* comm, const float* X, const double* y, int64_t n, int32_t dg,
                           int32_t max_depth, int64_t min_leaf, cudaStream_t s, dt_tree** out) {
  const int world = comm_world(comm), rank = comm_rank(comm);
  if (world > dg) return fail(DT_ERR_INVALID_ARG, "dt_fit_sharded: world must be <= d (feature sharding)");
  const int dloc = (dg - rank + world - 1) / world;
  Workspace ws;
  ws.s = s;
  FitBufs b{};
  auto get = [&](auto** p, size_t count) -> cudaError_t { return ws.get(p, count); };
  dt_status st = fit_alloc(b, n, dloc, max_depth, world, get);
  if (st != DT_OK) return st;
  std::vector<Pending> pending;
  st = fit_enqueue(b, X, y, n, dloc, max_depth, min_leaf, s, true, &pending, ShardCtx{comm, world, rank, dg});
  if (st != DT_OK) return st;
  return fit_finish(b, dg, s, &pending, out);
}

}  // namespace dtl
