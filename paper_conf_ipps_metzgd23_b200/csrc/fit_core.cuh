// Internal types of the level-synchronous exact CART fit (fit.cu, level.cu, presort.cu).
// Not part of the C ABI.  Method: PAPER.md:201-203 ("Decision Tree regression"); split
// rule, ties, thresholds and leaf rules: DESIGN.md Readings R1-R10, R19.
//
// Data layout on one rank, level l:
//   lists     the level's feature lists concatenated feature-major; list f holds, node
//             after node, this rank's entries of every searchable node, each node's run
//             sorted by (x_f, row id).  SoA: x f32, row u32, y (int32 when Reading R24
//             holds, else f64).  Double-buffered (level l is read while l+1 is written).
//   segments  (node k, feature f) runs of the lists: SegT[f * K + k] (start, local count,
//             and the rank carries of the value-range sharded fit: entries, S' and the
//             last x of the node's f-order held by lower ranks; zero / none for P = 1).
//   chunks    256 consecutive list entries (a warp's unit of work; lane L owns entries
//             8L .. 8L+7).  desc[chunk] = the segment of the chunk's first entry.
// One fused pass per level (level.cu, F_C) partitions the level-l lists into the
// children's level-(l+1) lists AND evaluates every split candidate of the children,
// with per-chunk carries from a fixed-shape scan of chunk aggregates (F_A, F_B), so
// every sum has a fixed association order (bit-reproducible; exact in integer mode).
#pragma once
#include <math.h>
#include <stdint.h>

#include "dt_internal.cuh"

namespace dtl {

constexpr int kItems = 8;                 // entries per lane
constexpr int kChunkW = 32 * kItems;      // entries per warp chunk
constexpr uint32_t kSmallSeg = 32;         // split segments of <= 32 entries: the small pass (warp per segment)
#ifndef DT_BLOCK_CHUNKS
#define DT_BLOCK_CHUNKS 256  // 1024 measured 0.6% slower per step (a deeper block scan)
#endif
constexpr int kBlockChunks = DT_BLOCK_CHUNKS;  // chunks per block of the chunk-carry scan (F_B) = its block size
constexpr int kMaxLogLevels = 4096;

// Per-level node (level-local index k).
struct NodeL {
  uint32_t N;          // rows of the node (global)
  int32_t id;          // BFS index in the output node array
  int32_t searchable;  // split search runs (depth < max_depth, N >= 2m)
  uint32_t parent;     // level-(l-1) index of the parent (root: 0)
  double c;            // centre (integer mode: floor(S/N); real mode: value)
  double sc;           // S' = sum over the node's rows of (y - c)
  double v;            // value = mean y
  uint32_t side;       // 0 = left child, 1 = right child (root: 0)
  uint32_t wstart;     // P = 1: first position of the node in every list of its level
  uint32_t pad[4];
};
static_assert(sizeof(NodeL) == 64, "NodeL layout");

struct SegT {
  uint64_t start;  // first position in the level's concatenated lists
  uint32_t cnt;    // this rank's entries
  uint32_t k;      // node
  int32_t f;       // feature (list) index
  uint32_t ioff;   // rank carry: entries of the node's global f-order on lower ranks
  double soff;     // rank carry: sum of (y - c_k) over those entries
  float xprev;     // rank carry: x of the last of those entries (NaN if ioff == 0)
  uint32_t pad;
};
static_assert(sizeof(SegT) == 40, "SegT layout");

constexpr uint32_t DEC_ALL_LEFT = 1u;  // virtual root pass: every row goes "left" (to the root)
struct Decision {
  int32_t f;       // split feature (global index), -1 = leaf
  uint32_t nl;     // rows going left (global)
  uint32_t kid;    // level-(l+1) index of the left child (right = kid + 1)
  uint32_t flags;
  double sl;       // S'_L (parent-centred) at the split
  double thr;      // threshold
};

// Per parent segment plan of the fused pass (built per level by tables_kernel).
constexpr uint32_t PS_SPLIT = 1u, PS_ALLLEFT = 2u, PS_SRCH0 = 4u, PS_SRCH1 = 8u, PS_WR0 = 16u, PS_WR1 = 32u;
struct __align__(16) PSeg {
  uint64_t start;      // parent segment in the level-l lists
  uint32_t cnt, k;
  int32_t f;
  uint32_t flags;
  uint32_t cs[2];      // child segment ids (level l+1)
  uint64_t ostart[2];  // child segment starts in the level-(l+1) lists
  double c[2], v[2], sc[2];  // children: centre, value, S'
  uint32_t N[2];       // children: rows (global)
  uint32_t ioff[2];    // children: rank carries (see SegT)
  double soff[2];
  float xprev[2];
  uint32_t kid;
  uint32_t glim;       // go-left bitmap: this rank's first glim entries of the segment go left
};
static_assert(sizeof(PSeg) == 144, "PSeg is copied with one bulk copy");

// Chunk aggregate of the fused pass: left count, child-centred sums of both sides, last x
// of both sides (NaN = none), since the last segment head of the chunk (flag).
struct AggP {
  uint32_t flag, nl;
  double sl, sr;
  float xl, xr;
};
static_assert(sizeof(AggP) == 32, "AggP layout");

__device__ __forceinline__ AggP agg_ident() {
  AggP a;
  a.flag = 0u;
  a.nl = 0u;
  a.sl = 0.0;
  a.sr = 0.0;
  a.xl = __int_as_float(0x7fc00000);
  a.xr = __int_as_float(0x7fc00000);
  return a;
}
__device__ __forceinline__ AggP combine(const AggP& a, const AggP& b) {
  if (b.flag) return b;
  AggP r;
  r.flag = a.flag;
  r.nl = a.nl + b.nl;
  r.sl = __dadd_rn(a.sl, b.sl);
  r.sr = __dadd_rn(a.sr, b.sr);
  r.xl = isnan(b.xl) ? a.xl : b.xl;
  r.xr = isnan(b.xr) ? a.xr : b.xr;
  return r;
}
__device__ __forceinline__ AggP shfl_up(const AggP& v, int delta) {
  AggP r;
  r.flag = __shfl_up_sync(0xffffffffu, v.flag, delta);
  r.nl = __shfl_up_sync(0xffffffffu, v.nl, delta);
  r.sl = __shfl_up_sync(0xffffffffu, v.sl, delta);
  r.sr = __shfl_up_sync(0xffffffffu, v.sr, delta);
  r.xl = __shfl_up_sync(0xffffffffu, v.xl, delta);
  r.xr = __shfl_up_sync(0xffffffffu, v.xr, delta);
  return r;
}
__device__ __forceinline__ AggP shfl_idx(const AggP& v, int src) {
  AggP r;
  r.flag = __shfl_sync(0xffffffffu, v.flag, src);
  r.nl = __shfl_sync(0xffffffffu, v.nl, src);
  r.sl = __shfl_sync(0xffffffffu, v.sl, src);
  r.sr = __shfl_sync(0xffffffffu, v.sr, src);
  r.xl = __shfl_sync(0xffffffffu, v.xl, src);
  r.xr = __shfl_sync(0xffffffffu, v.xr, src);
  return r;
}

// Split candidate piece: best of one (child segment, chunk) piece.
struct Cand2 {
  double gain;  // -1 = none
  double sl;    // S'_L (child-centred) at the position
  double thr;   // threshold
  uint32_t j;   // global left count of the child (first j rows go left)
  uint32_t sp;  // child segment id
  uint32_t level;
  uint32_t pad;
};
static_assert(sizeof(Cand2) == 40, "Cand2 layout");

struct Stat {
  double sse, ymin, ymax, s1;  // sum (y - v)^2, min, max, sum (y - c)
};

// Per-node result of one rank's local split search (exchanged across ranks).
struct ExchRec {
  double gain;  // -1 = no valid candidate on this rank
  double sl, thr;
  uint32_t j;
  int32_t gf;   // feature of the local best
  double sse, ymin, ymax, s1;  // node statistics from this rank's feature-0 entries
};
static_assert(sizeof(ExchRec) == 64, "ExchRec layout");

// Per (child, feature) boundary record of the value-range sharded fit (allgathered).
struct BndRec {
  uint32_t cnt;  // this rank's entries
  float xlast;   // x of the last of them (NaN if none)
  double s;      // sum of (y - c_child) over them
};

struct Ctl {
  unsigned long long T[2];   // entries of the level's lists, by level parity
  unsigned long long T0[2];  // entries of feature list 0
  uint32_t K[2];             // nodes at the level, by level parity
  uint32_t A2;               // P = 1: rows per list of the next level (written children)
  int32_t next_id;           // output nodes allocated so far
  int32_t next_id_prev;      // next_id before the current level's children (number -> children_kernel)
  int32_t int_mode;
  int32_t y32;               // the level lists hold y as int32 (Reading R24)
  int32_t max_depth_seen;
  int32_t nonfinite;
  int32_t all_integral;
  uint32_t ticket;
  uint32_t nsrch;            // searchable children of the current pass (0: statistics only)
  uint32_t nch_last;         // chunks processed by the last fused pass (its candidate pieces)
  uint32_t nfast;            // chunk plan of the pass: chunks inside one split segment,
  uint32_t ngen;             //   chunks with segment heads inside,
  uint32_t nunit;            //   split segment pieces of chunks (the fused pass),
  uint32_t nsmall;           //   split segments of at most 32 entries (the small pass)
  unsigned long long split_evals;
  double ysum, ymin, ymax, ysc;
};

struct LevelLog {  // per-level counts (algorithmic-byte accounting of the profiled path)
  unsigned long long T, T_next;
  uint32_t K, K_next;
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

__device__ __forceinline__ void neu_add(double& s, double& c, double v) {
  double t = __dadd_rn(s, v);
  if (fabs(s) >= fabs(v)) c = __dadd_rn(c, __dadd_rn(__dsub_rn(s, t), v));
  else c = __dadd_rn(c, __dadd_rn(__dsub_rn(v, t), s));
  s = t;
}

// Gain of candidate "first nl rows left" (Reading R19), no FMA contraction:
//   D = S'_L n_R - S'_R n_L,  gain = D^2 / ((N n_L) n_R).
__device__ __forceinline__ double split_gain_d(double sl, double sc, double nl, double Nd) {
  const double nr = __dsub_rn(Nd, nl);
  const double sr = __dsub_rn(sc, sl);
  const double D = __dsub_rn(__dmul_rn(sl, nr), __dmul_rn(sr, nl));
  return __ddiv_rn(__dmul_rn(D, D), __dmul_rn(__dmul_rn(Nd, nl), nr));
}

// The segment holding list position p: the largest t in [lo, hi] with segs[t].start <= p,
// given segs[lo].start <= p.  Segments tile the level's lists in index order and an empty
// segment shares its successor's start, so t is the non-empty segment containing p.
// Galloping from lo (the next few segments are the usual answer), then bisection: a walk
// over long runs of small or empty segments costs O(log distance) loads instead of O(distance).
template <class Seg>
__device__ __forceinline__ uint32_t seg_gallop(const Seg* __restrict__ segs, uint32_t lo, uint32_t hi, uint64_t p) {
  uint32_t step = 1u;
  while (lo < hi) {
    const uint32_t t = (hi - lo > step) ? lo + step : hi;
    if (__ldg(&segs[t].start) <= p) {
      lo = t;
      step <<= 1;
    } else {
      hi = t - 1u;
      break;
    }
  }
  while (lo < hi) {
    const uint32_t mid = lo + ((hi - lo + 1u) >> 1);
    if (__ldg(&segs[mid].start) <= p) lo = mid;
    else hi = mid - 1u;
  }
  return lo;
}

__device__ __forceinline__ double mid_threshold(float xlo, float xhi) {  // Reading R5
  return __dadd_rn(__ddiv_rn((double)xlo, 2.0), __ddiv_rn((double)xhi, 2.0));
}

// ---------------------------------------------------------------- fit buffers --------

struct FitBufs {
  float* lx[2];
  uint32_t* lr[2];
  double* ly[2];       // f64 or int32 entries (Reading R24)
  NodeL* nodes[2];
  SegT* segs[2];
  PSeg* pseg;
  Decision* dec;
  uint32_t* wst;  // number -> children_kernel: written-children offset per split node
  Decision* dec_root;  // the virtual-root decision (all rows to node 0)
  uint32_t* desc[2];
  AggP *agg, *cexcl, *bagg, *bcarry;
  AggP* tails;         // sharded: per parent segment, its aggregate from its last chunk
  uint8_t* gm;         // go-left bits per chunk entry (32 B per chunk)
  uint2* fast_list;    // chunk plan of the pass: {chunk, segment} inside one split segment
  uint32_t* gen_list;  // chunks with segment heads inside
  uint2* unit_list;    // {chunk, segment}: split segment pieces of chunks (fused pass)
  uint32_t* small_list;  // split segments of at most 32 entries (their ids)
  Cand2 *head_cand, *cont_cand;
  unsigned long long *slot_gain, *slot_pos;
  Stat *head_stat, *cont_stat;
  uint32_t* gbits;     // go-left bitmap over the (global) row ids
  int64_t nwords4;     // bitmap words (multiple of 4)
  dt_node* dout;
  Ctl* ctl;
  LevelLog* lvlog;
  // root statistics
  void* parts;
  double* cparts;
  int64_t root_np, root_chunk;
  // presort (keys / values alias the level-1 lists)
  uint32_t *k_in, *k_out, *v_in, *v_out;
  uint32_t *rs_cnt, *rs_off, *rs_tot;
  int rs_tiles;
  // sharded
  ExchRec *exch_send, *exch_all;
  BndRec *bnd_send, *bnd_all;
  unsigned long long* scan_tmp;  // block partials of the flat segment scan
  int64_t n, kcap, segcap, out_cap, max_chunks, max_cblocks;
  int d;
};

// Enqueue helpers across translation units.
dt_status presort_enqueue(const FitBufs& b, const float* X, const double* y, int64_t n, int d, int dg,
                          int64_t row0, int32_t max_depth, int64_t min_leaf, cudaStream_t s);
struct LevelArgs {
  int level;        // parent level (-1 = the virtual-root pass)
  int cur;          // list buffer holding the parent level
  int par;          // parity of the parent level's tables (level -1 uses level 0's)
  int d;            // lists (features) per level on this rank
  int64_t min_leaf;
  bool tails;       // sharded: per-segment tail aggregates
};
dt_status presort_sharded_enqueue(const FitBufs& b, dt_comm* comm, const float* X, const double* y, int64_t n_local,
                                  int64_t row0, int64_t n_global, int d, int32_t max_depth, int64_t min_leaf,
                                  cudaStream_t s);
dt_status forest_tree_enqueue(const FitBufs& b, const float* sx, const uint32_t* sr, const double* sy,
                              const double* y, int64_t n, int d, int32_t max_depth, int64_t min_leaf, uint64_t seed,
                              const uint32_t* tdev, int y32, uint32_t* w, double* ys, unsigned long long* tsum,
                              cudaStream_t s);
dt_status level_agg_enqueue(const FitBufs& b, const LevelArgs& la, cudaStream_t s);
dt_status level_fused_enqueue(const FitBufs& b, const LevelArgs& la, cudaStream_t s);

}  // namespace dtl
