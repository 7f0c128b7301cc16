// Exact greedy CART regression fit on B200 ("Decision Tree regression";
// split rule, tie rule, threshold and leaf rules: DESIGN.md Readings R1-R10, R19).
//
// Level-synchronous and exact (every feature, every threshold, every node); data layout
// and the fused per-level pass: fit_core.cuh, level.cu.  Per fit:
//   presort (presort.cu)  root statistics; per-feature stable sort of (x, row id) -> the
//                         level-0 lists; the virtual-root pass (F_A, F_B, F_C with every
//                         row "left" of a virtual parent) scores the root's candidates.
//   per level l:
//     piece_pos   lowest position among the candidate pieces holding each segment's best gain
//     select      per node: best feature (ties: lowest feature, then lowest position), node
//                 statistics, leaf rules, threshold -> decision + output node (a5, a8)
//     number      BFS numbering of the children, their exact statistics (a3)
//     tables      children's segment table, the level's per-segment plan
//     goleft      bit per row: 1 if the row goes left (a6)
//     F_A, F_B    chunk aggregates + carries (level.cu)
//     F_C         fused stable partition into the children's lists + the children's split
//                 search (a4, a7) (level.cu)
// No host synchronisation inside the level loop (counts live on the device).  Bounded-depth
// fits are captured once into a CUDA graph and replayed for repeated fits of the same inputs.
#include <math.h>
#include <stdio.h>

#include <algorithm>
#include <memory>
#include <mutex>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "fit_core.cuh"

namespace dtl {

namespace {
// NVTX ranges (presort, every level) for nsys / ncu --nvtx; no-ops without a tool attached
struct Nvtx {
  explicit Nvtx(const char* name) { nvtxRangePushA(name); }
  ~Nvtx() { nvtxRangePop(); }
};
}  // namespace

namespace {

// ----------------------------------------------------------------------------- select --

struct SelectArgs {
  uint4* gbits;  // go-left bitmap: zeroed here (grid-stride) for this level's goleft
  int64_t nvec;
  const NodeL* nodes;
  const SegT* segs_prev;  // the parent level's segments (statistics pieces); level 0: its own
  Ctl* ctl;
  int par;
  int level;
  int d;          // features (lists)
  const Cand2* head_cand;
  const Cand2* cont_cand;
  const Stat* head_stat;
  const Stat* cont_stat;
  Decision* dec;
  dt_node* out;
  LevelLog* log;
  unsigned long long* slot_gain;
  unsigned long long* slot_pos;
  ExchRec* exch;
  int world;
};

// Lowest position among the pieces whose gain equals their segment's maximum (the pieces
// were written by the previous F_C pass with an atomic max of the gain): key = j << 32 |
// piece location (bit 31: head piece).  Exact and order-independent.
__global__ void __launch_bounds__(256) piece_pos_kernel(const Ctl* __restrict__ ctl, int par, int d, uint32_t level,
                                                        const Cand2* __restrict__ head_cand,
                                                        const Cand2* __restrict__ cont_cand,
                                                        const unsigned long long* __restrict__ slot_gain,
                                                        unsigned long long* __restrict__ slot_pos) {
  const uint32_t K = ctl->K[par];
  const int64_t npc = 2 * (int64_t)ctl->nch_last;
  const int64_t nh = (int64_t)K * d;
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < npc + nh; r += (int64_t)gridDim.x * blockDim.x) {
    const bool head = r >= npc;
    const int64_t loc = head ? r - npc : r;
    const Cand2 c = head ? head_cand[loc] : cont_cand[loc];
    if (c.level != level || !(c.gain >= 0.0) || (int64_t)c.sp >= nh) continue;
    if ((unsigned long long)__double_as_longlong(c.gain) == slot_gain[c.sp])
      atomicMin(slot_pos + c.sp, ((unsigned long long)c.j << 32) | (unsigned long long)loc |
                                     (head ? 0x80000000ull : 0ull));
  }
}

__device__ __forceinline__ Cand2 piece_at(const SelectArgs& a, unsigned long long key) {
  const uint32_t loc = (uint32_t)key;
  return (loc & 0x80000000u) ? a.head_cand[loc & 0x7fffffffu] : a.cont_cand[loc];
}

// Leaf rules and the decision of node k from the ranks' records (fixed order: highest
// gain, then lowest feature, then lowest position; statistics combined in rank order).
// Identical inputs on every rank -> identical trees.
__device__ __forceinline__ void decide_node(const SelectArgs& a, uint32_t k, const NodeL& nd,
                                            const ExchRec* __restrict__ all, int64_t stride) {
  ExchRec st = all[k];
  for (int r = 1; r < a.world; ++r) {
    const ExchRec c = all[(int64_t)r * stride + k];
    st.sse = __dadd_rn(st.sse, c.sse);
    st.ymin = fmin(st.ymin, c.ymin);
    st.ymax = fmax(st.ymax, c.ymax);
    st.s1 = __dadd_rn(st.s1, c.s1);
  }
  const bool pure = !(st.ymin < st.ymax);
  int bf = -1;
  ExchRec best;
  best.gain = -1.0;
  best.j = 0;
  if (nd.searchable && !pure) {
    for (int r = 0; r < a.world; ++r) {
      const ExchRec c = all[(int64_t)r * stride + k];
      if (c.gain < 0.0) continue;
      if (bf < 0 || c.gain > best.gain || (c.gain == best.gain && (c.gf < bf || (c.gf == bf && c.j < best.j)))) {
        best = c;
        bf = c.gf;
      }
    }
    atomicAdd(&a.ctl->split_evals, (unsigned long long)nd.N * (unsigned long long)a.d);
  }
  Decision dc;
  dt_node o;
  o.depth = a.level;
  // value = mean of the node's rows.  Integer mode: exact fl(S/N) from the exact
  // bookkeeping.  Real mode: centre + fresh sum (y - c) / N, and exactly y for a pure
  // node (all rows equal), so single-row leaves reproduce their target.
  if (a.ctl->int_mode) o.value = nd.v;
  else o.value = pure ? st.ymin : __dadd_rn(nd.c, __ddiv_rn(st.s1, (double)nd.N));
  o.impurity = __ddiv_rn(st.sse, (double)nd.N);
  o.n_samples = nd.N;
  o.left = -1;
  o.right = -1;
  dc.kid = 0;
  dc.flags = 0;
  if (bf >= 0) {
    dc.f = bf;
    dc.nl = best.j;
    dc.sl = best.sl;
    dc.thr = best.thr;
    o.feature = bf;
    o.threshold = best.thr;
  } else {
    dc.f = -1;
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

// Statistics pieces of node k in index order (the F_C pass wrote one per chunk of its
// parent's feature-0 segment): the head piece, then one per later chunk.
__device__ __forceinline__ void stat_range(const SelectArgs& a, const NodeL& nd, int64_t& c0, int64_t& c1) {
  const SegT ps = a.segs_prev[nd.parent];  // feature 0 of the parent: index 0 * Kp + parent
  if (ps.cnt == 0) {
    c0 = 0;
    c1 = -1;
    return;
  }
  c0 = (int64_t)(ps.start / kChunkW);
  c1 = (int64_t)((ps.start + ps.cnt - 1) / kChunkW);
}
__device__ __forceinline__ void fold_stats(const SelectArgs& a, uint32_t k, uint32_t side, int64_t c0, int64_t lo,
                                           int64_t hi, Stat& acc) {
  for (int64_t b = lo; b < hi; b += 8) {
    Stat v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int64_t pc = b + u;
      if (pc < hi) v[u] = (pc == 0) ? a.head_stat[k] : a.cont_stat[2 * (c0 + pc) + side];
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

__device__ __forceinline__ ExchRec make_rec(const SelectArgs& a, int bf, unsigned long long key, const Stat& st) {
  ExchRec r;
  r.gain = -1.0;
  r.sl = 0.0;
  r.thr = 0.0;
  r.j = 0;
  r.gf = -1;
  if (bf >= 0) {
    const Cand2 c = piece_at(a, key);
    r.gain = c.gain;
    r.sl = c.sl;
    r.thr = c.thr;
    r.j = c.j;
    r.gf = bf;
  }
  r.sse = st.sse;
  r.ymin = st.ymin;
  r.ymax = st.ymax;
  r.s1 = st.s1;
  return r;
}

__global__ void __launch_bounds__(256) select_kernel(SelectArgs a) {
  const uint32_t K = a.ctl->K[a.par];
  __shared__ double s_gain[256];
  __shared__ unsigned long long s_key[256];
  __shared__ Stat s_stat[256];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  // nothing reads the bitmap between the previous level's F_A and this level's goleft
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + tid; i < a.nvec; i += (int64_t)gridDim.x * blockDim.x)
    a.gbits[i] = make_uint4(0u, 0u, 0u, 0u);
  if (blockIdx.x == 0 && tid == 0) a.ctl->nfast = a.ctl->ngen = a.ctl->nunit = a.ctl->nsmall = 0u;  // next chunk plan
  if (blockIdx.x == 0 && tid == 0 && a.level < kMaxLogLevels) {
    a.log[a.level].T = a.ctl->T[a.par];
    a.log[a.level].K = K;
    a.log[a.level].T_next = 0;
    a.log[a.level].K_next = 0;
  }
  if (K > gridDim.x / 4) {
    // many (small) nodes: one warp per node, no block barriers
    const int nwarps = blockDim.x >> 5;
    for (uint32_t k = blockIdx.x * nwarps + w; k < K; k += gridDim.x * nwarps) {
      const NodeL nd = a.nodes[k];
      double bg = -1.0;
      unsigned long long bkey = ~0ull;
      int bf = 0x7fffffff;
      for (int f = lane; f < a.d; f += 32) {
        const int64_t s = (int64_t)f * K + k;
        if (nd.searchable) {
          const unsigned long long key = a.slot_pos[s];
          if (key != ~0ull) {
            const double g = __longlong_as_double((long long)a.slot_gain[s]);
            if (g > bg) { bg = g; bkey = key; bf = f; }  // strict >: lowest feature of this lane
          }
        }
        a.slot_gain[s] = 0ull;
        a.slot_pos[s] = ~0ull;
      }
      double gmax = bg;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) gmax = fmax(gmax, __shfl_xor_sync(0xffffffffu, gmax, off));
      const int wf = __reduce_min_sync(0xffffffffu, (bg == gmax && bg >= 0.0) ? bf : 0x7fffffff);
      const int src = __ffs(__ballot_sync(0xffffffffu, bf == wf)) - 1;
      const unsigned long long wkey = __shfl_sync(0xffffffffu, bkey, src < 0 ? 0 : src);
      int64_t c0, c1;
      stat_range(a, nd, c0, c1);
      const int64_t np = c1 - c0 + 1;
      const int64_t per = (np + 31) / 32;
      Stat acc{0.0, INFINITY, -INFINITY, 0.0};
      fold_stats(a, k, nd.side, c0, lane * per, min(np, (lane + 1) * per), acc);
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
        a.exch[k] = make_rec(a, wf != 0x7fffffff ? wf : -1, wkey, acc);
        if (a.world == 1) decide_node(a, k, nd, a.exch, 0);  // single rank: decide in place
      }
    }
    return;
  }
  for (uint32_t k = blockIdx.x; k < K; k += gridDim.x) {
    const NodeL nd = a.nodes[k];
    for (int f = tid; f < a.d; f += blockDim.x) {
      const int64_t s = (int64_t)f * K + k;
      double bg = -1.0;
      unsigned long long key = ~0ull;
      if (nd.searchable) {
        key = a.slot_pos[s];
        if (key != ~0ull) bg = __longlong_as_double((long long)a.slot_gain[s]);
      }
      a.slot_gain[s] = 0ull;
      a.slot_pos[s] = ~0ull;
      s_gain[f] = bg;
      s_key[f] = key;
    }
    {
      int64_t c0, c1;
      stat_range(a, nd, c0, c1);
      const int64_t np = c1 - c0 + 1;
      const int64_t per = (np + blockDim.x - 1) / blockDim.x;
      Stat acc{0.0, INFINITY, -INFINITY, 0.0};
      fold_stats(a, k, nd.side, c0, tid * per, min(np, (tid + 1) * per), acc);
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
      int bf = -1;
      double bg = -1.0;
      for (int f = 0; f < a.d; ++f)
        if (s_gain[f] > bg) { bg = s_gain[f]; bf = f; }  // strict >: lowest feature wins ties
      a.exch[k] = make_rec(a, bf, bf >= 0 ? s_key[bf] : ~0ull, s_stat[0]);
      if (a.world == 1) decide_node(a, k, nd, a.exch, 0);
    }
    __syncthreads();
  }
}

__global__ void __launch_bounds__(256) decide_kernel(SelectArgs a, const ExchRec* __restrict__ all, int64_t stride) {
  const uint32_t K = a.ctl->K[a.par];
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < K; k += gridDim.x * blockDim.x)
    decide_node(a, k, a.nodes[k], all, stride);
}

// ----------------------------------------------------------------------------- number --

struct NumberArgs {
  const NodeL* nodes;
  NodeL* next;
  Decision* dec;
  Ctl* ctl;
  int par;
  int level;
  int d;
  int32_t max_depth;
  int64_t min_leaf;
  dt_node* out;
  LevelLog* log;
  uint32_t* wst;  // per split node: its written children's first position (scan -> children_kernel)
};

// Single block: BFS numbering (children appended left, right in node order) and (P = 1)
// the children's positions in the next level's lists (written children = searchable
// children, in node order): three block scans over the nodes.  children_kernel then
// builds the children (exact statistics) on the whole grid.
__global__ void __launch_bounds__(1024) number_kernel(NumberArgs a) {
  __shared__ unsigned long long sh_a[33], sh_b[33], sh_c[33];
  __shared__ unsigned long long base_split, base_rows, base_srch;
  const uint32_t K = a.ctl->K[a.par];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const int next_id0 = a.ctl->next_id;
  const int child_depth = a.level + 1;
  const bool depth_ok = (a.max_depth < 0) || (child_depth < a.max_depth);
  if (tid == 0) { base_split = 0; base_rows = 0; base_srch = 0; }
  __syncthreads();
  for (uint32_t k0 = 0; k0 < K; k0 += blockDim.x) {
    const uint32_t k = k0 + tid;
    const bool in = k < K;
    const Decision dc = in ? a.dec[k] : Decision{-1, 0, 0, 0, 0.0, 0.0};
    const uint32_t nN = in ? a.nodes[k].N : 0u;  // loaded beside the decision (no dependent load)
    const bool sp = in && dc.f >= 0;
    const uint32_t nl = sp ? dc.nl : 0u, nr = sp ? nN - dc.nl : 0u;
    const bool sl_ok = sp && depth_ok && (int64_t)nl >= 2 * a.min_leaf;
    const bool sr_ok = sp && depth_ok && (int64_t)nr >= 2 * a.min_leaf;
    // three exclusive scans over the block: splits, written rows, searchable children
    const unsigned long long va = sp ? 1ull : 0ull, vb = (sl_ok ? nl : 0ull) + (sr_ok ? nr : 0ull),
                             vc = (sl_ok ? 1ull : 0ull) + (sr_ok ? 1ull : 0ull);
    unsigned long long ia = va, ib = vb, ic = vc;
#pragma unroll
    for (int dd = 1; dd < 32; dd <<= 1) {
      const unsigned long long oa = __shfl_up_sync(0xffffffffu, ia, dd);
      const unsigned long long ob = __shfl_up_sync(0xffffffffu, ib, dd);
      const unsigned long long oc = __shfl_up_sync(0xffffffffu, ic, dd);
      if (lane >= dd) { ia += oa; ib += ob; ic += oc; }
    }
    if (lane == 31) { sh_a[w] = ia; sh_b[w] = ib; sh_c[w] = ic; }
    __syncthreads();
    if (w == 0) {  // the 32 warp totals: exclusive prefixes (and the tile totals in [32])
      const unsigned long long ta = sh_a[lane], tb = sh_b[lane], tc = sh_c[lane];
      unsigned long long xa = ta, xb = tb, xc = tc;
#pragma unroll
      for (int dd = 1; dd < 32; dd <<= 1) {
        const unsigned long long oa = __shfl_up_sync(0xffffffffu, xa, dd);
        const unsigned long long ob = __shfl_up_sync(0xffffffffu, xb, dd);
        const unsigned long long oc = __shfl_up_sync(0xffffffffu, xc, dd);
        if (lane >= dd) { xa += oa; xb += ob; xc += oc; }
      }
      sh_a[lane] = xa - ta; sh_b[lane] = xb - tb; sh_c[lane] = xc - tc;
      if (lane == 31) { sh_a[32] = xa; sh_b[32] = xb; sh_c[32] = xc; }
    }
    __syncthreads();
    const uint32_t rank = (uint32_t)(base_split + sh_a[w] + (ia - va));
    const unsigned long long rows_ex = base_rows + sh_b[w] + (ib - vb);
    if (sp) {
      Decision d2 = dc;
      d2.kid = 2 * rank;
      a.dec[k] = d2;
      a.wst[k] = (uint32_t)rows_ex;
    }
    __syncthreads();
    if (tid == 0) { base_split += sh_a[32]; base_rows += sh_b[32]; base_srch += sh_c[32]; }
    __syncthreads();
  }
  if (tid == 0) {
    const int np = a.par ^ 1;
    a.ctl->next_id_prev = next_id0;
    a.ctl->K[np] = (uint32_t)(2 * base_split);
    a.ctl->A2 = (uint32_t)base_rows;
    a.ctl->T[np] = base_rows * (unsigned long long)a.d;
    a.ctl->T0[np] = base_rows;
    a.ctl->nsrch = (uint32_t)base_srch;
    a.ctl->next_id = next_id0 + 2 * (int)base_split;
    if (a.level < kMaxLogLevels) {
      a.log[a.level].T_next = base_rows * (unsigned long long)a.d;
      a.log[a.level].K_next = (uint32_t)(2 * base_split);
    }
  }
}

// The children of every split node (grid-stride): ids, exact statistics (Reading R17 /
// real mode), searchability, list positions; the parent's child links.
__global__ void __launch_bounds__(256) children_kernel(NumberArgs a) {
  const uint32_t K = a.ctl->K[a.par];
  const int next_id0 = a.ctl->next_id_prev;
  const int int_mode = a.ctl->int_mode;
  const int child_depth = a.level + 1;
  const bool depth_ok = (a.max_depth < 0) || (child_depth < a.max_depth);
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < K; k += gridDim.x * blockDim.x) {
    // the decision, the node and its row offset loaded together (no dependent loads)
    const Decision dc = a.dec[k];
    const NodeL nd = a.nodes[k];
    const unsigned long long rows_ex = a.wst[k];
    if (dc.f < 0) continue;
    const uint32_t rank = dc.kid >> 1;
    const uint32_t nl = dc.nl, nr = nd.N - dc.nl;
    const bool sl_ok = depth_ok && (int64_t)nl >= 2 * a.min_leaf;
    const bool sr_ok = depth_ok && (int64_t)nr >= 2 * a.min_leaf;
    const int lid = next_id0 + 2 * (int)rank;
    a.out[nd.id].left = lid;
    a.out[nd.id].right = lid + 1;
    NodeL L, R;
    L.N = nl;
    R.N = nr;
    L.id = lid;
    R.id = lid + 1;
    L.searchable = sl_ok ? 1 : 0;
    R.searchable = sr_ok ? 1 : 0;
    L.parent = R.parent = k;
    L.side = 0;
    R.side = 1;
    L.wstart = (uint32_t)rows_ex;
    R.wstart = (uint32_t)(rows_ex + (sl_ok ? nl : 0u));
    L.pad[0] = L.pad[1] = L.pad[2] = L.pad[3] = 0;
    R.pad[0] = R.pad[1] = R.pad[2] = R.pad[3] = 0;
    const double slp = dc.sl;                  // parent-centred S'_L
    const double srp = __dsub_rn(nd.sc, slp);  // parent-centred S'_R
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
  }
}

// ----------------------------------------------------------------------------- goleft --

// Bit per row: 1 if the row goes to its node's left child -- the first nl entries of the
// node's split-feature list (a6).  Each thread tests one chunk of the level's lists (does
// it hold left entries of a split feature?); the warp then sets the bits of the
// qualifying chunks together.
__global__ void __launch_bounds__(256) goleft_kernel(const Ctl* __restrict__ ctl, int par, const uint32_t* __restrict__ desc,
                                                     const PSeg* __restrict__ pseg, const uint32_t* __restrict__ lr,
                                                     uint32_t* __restrict__ gbits, int d) {
  const uint64_t T = ctl->T[par];
  if (ctl->K[par ^ 1] == 0) return;  // nothing splits
  const uint32_t nseg = ctl->K[par] * (uint32_t)d;
  const int64_t nch = (int64_t)((T + kChunkW - 1) / kChunkW);
  const int lane = threadIdx.x & 31;
  // warp gw tests chunks gw + (32 it + lane) nw: qualifying chunks (contiguous runs of a
  // split feature's list) spread over all warps
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t it = 0; gw + it * 32 * nw < nch; ++it) {
    const int64_t mych = gw + (it * 32 + lane) * nw;
    bool q = false;
    if (mych < nch) {
      const uint64_t cbase = (uint64_t)mych * kChunkW;
      const uint32_t s = __ldg(desc + mych);
      const uint64_t st = __ldg(&pseg[s].start), en = st + __ldg(&pseg[s].cnt);
      // one segment: does it hold left entries here?  Else segment heads inside: walk it
      q = (st <= cbase && en >= cbase + kChunkW) ? cbase < st + __ldg(&pseg[s].glim) : true;
    }
    uint32_t qm = __ballot_sync(0xffffffffu, q);
    while (qm) {
      const int c = __ffs(qm) - 1;
      qm &= qm - 1u;
      const int64_t ch = gw + (it * 32 + c) * nw;
      const uint64_t cbase = (uint64_t)ch * kChunkW;
      uint32_t s = __ldg(desc + ch);
      uint64_t st = __ldg(&pseg[s].start), en = st + __ldg(&pseg[s].cnt);
      uint64_t lim = st + __ldg(&pseg[s].glim);  // the segment's left entries: [st, lim)
      if (st <= cbase && en >= cbase + kChunkW) {
        // one segment (rows read coalesced)
        // every row id in flight first, then the bit updates (no load -> atomic chain)
        uint32_t rr[kItems];
#pragma unroll
        for (int j = 0; j < kItems; ++j) {
          const uint64_t p = cbase + (uint64_t)(j * 32 + lane);
          rr[j] = p < lim ? __ldg(lr + p) : 0xffffffffu;
        }
#pragma unroll
        for (int j = 0; j < kItems; ++j)
          if (rr[j] != 0xffffffffu) atomicOr(gbits + (rr[j] >> 5), 1u << (rr[j] & 31));
        continue;
      }
      // segment heads inside: lane owns entries 8 lane .. 8 lane + 7, finds their segments
      const uint64_t p0 = cbase + (uint64_t)(lane * kItems);
      uint32_t rr[kItems];
#pragma unroll
      for (int j = 0; j < kItems; ++j) rr[j] = 0xffffffffu;
#pragma unroll
      for (int j = 0; j < kItems; ++j) {
        const uint64_t p = p0 + j;
        if (p >= T) break;
        if (p >= en) {
          s = seg_gallop(pseg, s + 1u, nseg - 1u, p);
          st = __ldg(&pseg[s].start);
          en = st + __ldg(&pseg[s].cnt);
          lim = st + __ldg(&pseg[s].glim);
        }
        if (p < lim) rr[j] = __ldg(lr + p);
      }
#pragma unroll
      for (int j = 0; j < kItems; ++j)
        if (rr[j] != 0xffffffffu) atomicOr(gbits + (rr[j] >> 5), 1u << (rr[j] & 31));
    }
  }
}

// ----------------------------------------------------------------------------- tables --

// P = 1: the children's segment table (level l+1; written children at wstart of every
// list) and the plan of every level-l segment (children, centres, positions).
// mode 0 (P = 1): as above.  Sharded: mode 1 = the plans without the children's positions
// and rank carries (before the boundary exchange), mode 2 = those from segs_next.
// The fused pass's work on split segment [start, start + cnt) (levels >= 0; listed from
// the segment side): a segment of at most kSmallSeg entries -> the small list
// (fused_small_kernel); else the chunks it meets without covering them -- its first and
// last at most, the ones it covers are fast chunks (chunk_plan_kernel) -> unit-list pieces.
__device__ __forceinline__ void piece_chunks(uint64_t start, uint32_t cnt, uint32_t& u0, uint32_t& u1, uint32_t& sm) {
  if (cnt <= kSmallSeg) {
    sm = 0u;
    return;
  }
  const uint64_t end = start + cnt;
  const uint64_t c0 = start / kChunkW, c1 = (end - 1) / kChunkW;
  if (!(start == c0 * kChunkW && end >= c0 * kChunkW + kChunkW)) u0 = (uint32_t)c0;
  if (c1 > c0 && end < c1 * kChunkW + kChunkW) u1 = (uint32_t)c1;
}

__global__ void __launch_bounds__(256) tables_kernel(Ctl* __restrict__ ctl, int par, int d,
                                                     const NodeL* __restrict__ next, const Decision* __restrict__ dec,
                                                     const SegT* __restrict__ segs, SegT* __restrict__ segs_next,
                                                     PSeg* __restrict__ pseg, int mode, uint2* __restrict__ unit_list,
                                                     uint32_t* __restrict__ small_list) {
  const uint32_t K = ctl->K[par], K2 = ctl->K[par ^ 1];
  const uint64_t A2 = ctl->A2;
  if (mode == 2) {
    for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < (int64_t)K * d;
         s += (int64_t)gridDim.x * blockDim.x) {
      const uint32_t k = (uint32_t)(s % K);
      const Decision dc = dec[k];
      if (dc.f < 0) continue;
      const int f = (int)(s / K);
      for (int q = 0; q < 2; ++q) {
        const SegT c = segs_next[(int64_t)f * K2 + dc.kid + q];
        pseg[s].ostart[q] = c.start;
        pseg[s].ioff[q] = c.ioff;
        pseg[s].soff[q] = c.soff;
        pseg[s].xprev[q] = c.xprev;
      }
    }
    return;
  }
  const int64_t n1 = mode == 0 ? (int64_t)K2 * d : 0, n2 = (int64_t)K * d;
  const bool full = ctl->nsrch > 0;  // children searched: every list; else feature 0 (statistics)
  const int lane = threadIdx.x & 31;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n1 + n2; base += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = base + threadIdx.x;  // warp-uniform trip count (the appends below)
    uint32_t u0 = 0xffffffffu, u1 = 0xffffffffu, sm = 0xffffffffu;  // this segment's pieces
    if (i < n1) {
      const int f = (int)(i / K2);
      const uint32_t kc = (uint32_t)(i - (int64_t)f * K2);
      const NodeL c = next[kc];
      SegT sg;
      sg.start = (uint64_t)f * A2 + c.wstart;
      sg.cnt = c.searchable ? c.N : 0u;
      sg.k = kc;
      sg.f = f;
      sg.ioff = 0;
      sg.soff = 0.0;
      sg.xprev = __int_as_float(0x7fc00000);
      sg.pad = 0;
      segs_next[i] = sg;
    } else if (i < n1 + n2) {
      const int64_t s = i - n1;
      const int f = (int)(s / K);
      const uint32_t k = (uint32_t)(s - (int64_t)f * K);
      const SegT sg = segs[s];
      const Decision dc = dec[k];
      PSeg p;
      p.start = sg.start;
      p.cnt = sg.cnt;
      p.k = k;
      p.f = f;
      p.flags = 0;
      p.kid = 0;
      p.glim = 0;
      for (int q = 0; q < 2; ++q) {
        p.cs[q] = 0;
        p.ostart[q] = 0;
        p.c[q] = p.v[q] = p.sc[q] = p.soff[q] = 0.0;
        p.N[q] = p.ioff[q] = 0;
        p.xprev[q] = __int_as_float(0x7fc00000);
      }
      if (dc.f >= 0) {
        p.flags = PS_SPLIT;
        p.kid = dc.kid;
        if (dc.f == f) p.glim = min(sg.cnt, dc.nl > sg.ioff ? dc.nl - sg.ioff : 0u);
        for (int q = 0; q < 2; ++q) {
          const uint32_t kc = dc.kid + q;
          const NodeL c = next[kc];
          p.cs[q] = (uint32_t)((int64_t)f * K2 + kc);
          p.ostart[q] = (uint64_t)f * A2 + c.wstart;
          p.c[q] = c.c;
          p.v[q] = c.v;
          p.sc[q] = c.sc;
          p.N[q] = c.N;
          if (c.searchable) p.flags |= (q == 0 ? (PS_SRCH0 | PS_WR0) : (PS_SRCH1 | PS_WR1));
        }
      }
      pseg[s] = p;
      if ((p.flags & PS_SPLIT) && p.cnt && (full || f == 0)) piece_chunks(p.start, p.cnt, u0, u1, sm);
    }
    // warp-aggregated appends: pieces -> unit list, small segments -> small list
    const uint32_t lt = (1u << lane) - 1u;
    const uint32_t b0 = __ballot_sync(0xffffffffu, u0 != 0xffffffffu), b1 = __ballot_sync(0xffffffffu, u1 != 0xffffffffu);
    const uint32_t bs = __ballot_sync(0xffffffffu, sm != 0xffffffffu);
    uint32_t pu = 0, ps = 0;
    if (lane == 0) {
      if (b0 | b1) pu = atomicAdd(&ctl->nunit, (uint32_t)(__popc(b0) + __popc(b1)));
      if (bs) ps = atomicAdd(&ctl->nsmall, (uint32_t)__popc(bs));
    }
    pu = __shfl_sync(0xffffffffu, pu, 0) + __popc(b0 & lt) + __popc(b1 & lt);
    ps = __shfl_sync(0xffffffffu, ps, 0) + __popc(bs & lt);
    const uint32_t sid = (uint32_t)(i - n1);
    if (u0 != 0xffffffffu) unit_list[pu++] = make_uint2(u0, sid);
    if (u1 != 0xffffffffu) unit_list[pu] = make_uint2(u1, sid);
    if (sm != 0xffffffffu) small_list[ps] = sid;
  }
}

// ----------------------------------------------------------------------------- sharded --

// Value-range sharded fit: this rank's part of every child segment (count, last x, sum of
// (y - c_child)) from its parent segment's total aggregate = chunk carry of the segment's
// last chunk + that chunk's tail piece (F_A).
__global__ void __launch_bounds__(256) bnd_kernel(const Ctl* __restrict__ ctl, int par, int d,
                                                  const PSeg* __restrict__ pseg, const AggP* __restrict__ tails,
                                                  const AggP* __restrict__ cexcl, const AggP* __restrict__ bcarry,
                                                  BndRec* __restrict__ out) {
  const uint32_t K = ctl->K[par], K2 = ctl->K[par ^ 1];
  for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < (int64_t)K * d;
       s += (int64_t)gridDim.x * blockDim.x) {
    const PSeg ps = pseg[s];
    if (!(ps.flags & PS_SPLIT)) continue;
    BndRec L{0u, __int_as_float(0x7fc00000), 0.0}, R = L;
    if (ps.cnt) {
      const uint64_t last = ps.start + ps.cnt - 1;
      const int64_t c = (int64_t)(last / kChunkW);
      AggP t = tails[s];
      if (!t.flag) t = combine(combine(bcarry[c / kBlockChunks], cexcl[c]), t);
      L.cnt = t.nl;
      L.xlast = t.xl;
      L.s = t.sl;
      R.cnt = ps.cnt - t.nl;
      R.xlast = t.xr;
      R.s = t.sr;
    }
    const int64_t i = (int64_t)ps.f * K2 + ps.kid;
    out[i] = L;
    out[i + 1] = R;
  }
  (void)d;
}

// Flat exclusive scan of the children's written local counts over (feature, child) in
// feature-major order (the next level's list layout): block scans + block totals, the
// last block scans the totals (ticket).
__global__ void __launch_bounds__(1024) segscan_kernel(Ctl* ctl, int par, int d, const NodeL* __restrict__ next,
                                                       const BndRec* __restrict__ mine,
                                                       unsigned long long* __restrict__ excl,
                                                       unsigned long long* __restrict__ btot) {
  __shared__ unsigned long long sh[33];
  __shared__ bool s_last;
  const uint32_t K2 = ctl->K[par ^ 1];
  const int64_t n = (int64_t)K2 * d;
  const int64_t i = (int64_t)blockIdx.x * 1024 + threadIdx.x;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  unsigned long long v = 0;
  if (i < n) {
    const uint32_t kc = (uint32_t)(i % K2);
    v = next[kc].searchable ? mine[i].cnt : 0u;
  }
  unsigned long long inc = v;
#pragma unroll
  for (int dd = 1; dd < 32; dd <<= 1) {
    const unsigned long long o = __shfl_up_sync(0xffffffffu, inc, dd);
    if (lane >= dd) inc += o;
  }
  if (lane == 31) sh[w] = inc;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long r = 0;
    for (int q = 0; q < 32; ++q) { const unsigned long long t = sh[q]; sh[q] = r; r += t; }
    sh[32] = r;
  }
  __syncthreads();
  if (i < n) excl[i] = sh[w] + inc - v;
  if (threadIdx.x == 0) btot[blockIdx.x] = sh[32];
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) s_last = atomicAdd(&ctl->ticket, 1u) == gridDim.x - 1;
  __syncthreads();
  if (!s_last || threadIdx.x != 0) return;
  __threadfence();
  ctl->ticket = 0u;
  const int64_t nb = (n + 1023) / 1024;
  unsigned long long r = 0;
  for (int64_t b = 0; b < nb; ++b) {  // block offsets (in place), then the totals
    const unsigned long long t = __ldcg(btot + b);
    btot[b] = r;
    r += t;
  }
  ctl->T[par ^ 1] = r;
  (void)d;
}

// The next level's segment table: positions from the scan, rank carries from the ranks'
// records (rank order); the list sizes.
__global__ void __launch_bounds__(256) segwrite_kernel(Ctl* ctl, int par, int d, int rank, const NodeL* __restrict__ next,
                                                       const BndRec* __restrict__ all,
                                                       const unsigned long long* __restrict__ excl,
                                                       const unsigned long long* __restrict__ boff,
                                                       SegT* __restrict__ segs_next) {
  const uint32_t K2 = ctl->K[par ^ 1];
  const int64_t n = (int64_t)K2 * d;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t kc = (uint32_t)(i % K2);
    const int f = (int)(i / K2);
    uint32_t ioff = 0;
    double soff = 0.0;
    float xprev = __int_as_float(0x7fc00000);
    for (int q = 0; q < rank; ++q) {
      const BndRec r = all[(int64_t)q * n + i];
      ioff += r.cnt;
      soff = __dadd_rn(soff, r.s);
      if (r.cnt) xprev = r.xlast;
    }
    SegT sg;
    sg.start = boff[i / 1024] + excl[i];
    sg.cnt = next[kc].searchable ? all[(int64_t)rank * n + i].cnt : 0u;
    sg.k = kc;
    sg.f = f;
    sg.ioff = ioff;
    sg.soff = soff;
    sg.xprev = xprev;
    sg.pad = 0;
    segs_next[i] = sg;
    if (i == K2) ctl->T0[par ^ 1] = sg.start;  // feature list 0 ends where list 1 starts
  }
  if (blockIdx.x == 0 && threadIdx.x == 0 && d == 1) ctl->T0[par ^ 1] = ctl->T[par ^ 1];
}

// ----------------------------------------------------------------------------- finish --

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

__global__ void set_u32_kernel(uint32_t* p, uint32_t v) { *p = v; }

// ----------------------------------------------------------------------------- buffers --

struct Workspace {
  std::vector<void*> ptrs;
  cudaStream_t s;
  ~Workspace() {
    for (void* p : ptrs) cudaFreeAsync(p, s);
  }
  template <class T>
  cudaError_t get(T** p, size_t count) {
    cudaError_t e = cudaMallocAsync((void**)p, sizeof(T) * (count ? count : 1), s);
    if (e == cudaSuccess) ptrs.push_back(*p);
    return e;
  }
};

dt_status alloc_status(cudaError_t e) {
  if (e == cudaSuccess) return DT_OK;
  (void)cudaGetLastError();  // a failed allocation is not sticky: do not leak it into the next call
  return e == cudaErrorMemoryAllocation ? fail(DT_ERR_OOM, "dt_fit: device memory exhausted")
                                        : cuda_fail(e, "allocation", __FILE__, __LINE__);
}

// Allocates every buffer through `get` (stream-ordered or persistent).  n: this rank's
// rows (lists hold n * d entries), n_global: all ranks' rows (bitmap, node capacity).
template <class Get>
dt_status fit_alloc(FitBufs& b, int64_t n, int64_t n_global, int32_t d, int32_t max_depth, int64_t min_leaf,
                    int world, Get get) {
  const int64_t total0 = n * (int64_t)d;
  b.n = n;
  b.d = d;
  // nodes at a level: <= n_global / min_leaf (every node of level >= 1 is a child of a
  // split node with >= 2m rows), <= 2^depth
  b.kcap = std::max<int64_t>(1, (n_global + min_leaf - 1) / min_leaf);
  if (max_depth >= 0 && max_depth < 40) b.kcap = std::min<int64_t>(b.kcap, (int64_t)1 << max_depth);
  b.segcap = b.kcap * d;
  b.out_cap = 2 * n_global - 1;
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
  const size_t lcap = (size_t)total0 + kChunkW;  // + one chunk: bulk copies of a partial last chunk
#define GET(p, n_)                                           \
  do {                                                       \
    dt_status st__ = alloc_status(get(&(p), (size_t)(n_)));  \
    if (st__ != DT_OK) return st__;                          \
  } while (0)
  for (int k = 0; k < 2; ++k) {
    GET(b.lx[k], lcap);
    GET(b.lr[k], lcap);
    GET(b.ly[k], lcap);
    GET(b.nodes[k], b.kcap + 1);
    GET(b.segs[k], b.segcap);
    GET(b.desc[k], b.max_chunks);
  }
  GET(b.pseg, b.segcap);
  GET(b.dec, b.kcap);
  GET(b.wst, b.kcap);
  GET(b.dec_root, 1);
  GET(b.agg, b.max_chunks);
  GET(b.cexcl, b.max_chunks);
  GET(b.bagg, b.max_cblocks);
  GET(b.bcarry, b.max_cblocks);
  GET(b.gm, b.max_chunks * 32);
  GET(b.gen_list, b.max_chunks);
  GET(b.fast_list, b.max_chunks);
  GET(b.unit_list, b.max_chunks * 9);  // <= 9 pieces per listed chunk (kMaxPieces, level.cu)
  GET(b.small_list, b.segcap);
  GET(b.head_cand, b.segcap);
  GET(b.cont_cand, 2 * b.max_chunks);
  GET(b.slot_gain, b.segcap);
  GET(b.slot_pos, b.segcap);
  GET(b.head_stat, b.kcap);
  GET(b.cont_stat, 2 * b.max_chunks);
  b.nwords4 = ((n_global + 127) / 128) * 4;  // whole uint4s
  GET(b.gbits, b.nwords4);
  GET(b.dout, b.out_cap);
  GET(b.ctl, 1);
  GET(b.lvlog, kMaxLogLevels);
  {
    double* p = nullptr;
    GET(p, b.root_np * 6);  // RootPart (presort.cu): 6 words
    b.parts = p;
  }
  GET(b.cparts, b.root_np);
  // the presort's key / row buffers live in the level-1 lists (16 B per entry = exactly
  // the four 4-B arrays, with the f64 y list): dead once the level-0 lists are built,
  // before the first partition writes lists[1].  Saves 16 B per entry (C3: 51 GB).
  b.k_in = reinterpret_cast<uint32_t*>(b.lx[1]);
  b.k_out = b.lr[1];
  b.v_in = reinterpret_cast<uint32_t*>(b.ly[1]);
  b.v_out = reinterpret_cast<uint32_t*>(b.ly[1]) + total0;
  b.rs_tiles = (int)((n + 2047) / 2048);
  GET(b.rs_cnt, (size_t)d * 256 * b.rs_tiles);
  GET(b.rs_off, (size_t)d * 256 * b.rs_tiles);
  GET(b.rs_tot, (size_t)d * 256);
  b.tails = nullptr;
  b.bnd_send = b.bnd_all = nullptr;
  b.scan_tmp = nullptr;
  GET(b.exch_send, b.kcap);
  if (world > 1) {
    GET(b.exch_all, b.kcap * world);
    GET(b.tails, b.segcap);
    GET(b.bnd_send, 2 * b.segcap);
    GET(b.bnd_all, 2 * b.segcap * world);
    GET(b.scan_tmp, b.segcap + b.segcap / 1024 + 2);  // exclusive values, then block totals
  } else {
    b.exch_all = b.exch_send;
  }
#undef GET
  return DT_OK;
}

// profiling records whose bytes depend on device-side counts
struct Pending {
  int rec, level, kind;
};

int grid_of(const void* kern, int threads, size_t smem) {
  int per = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, kern, threads, smem);
  if (per < 1) per = 1;
  return num_sms() * per;
}

// Enqueues the whole fit on stream s (no host synchronisation unless `poll`).
dt_status fit_levels(const FitBufs& b, int32_t d, int32_t max_depth, int64_t min_leaf, cudaStream_t s, bool poll,
                     std::vector<Pending>* pending);

dt_status clear_pieces(const FitBufs& b, cudaStream_t s) {
  DT_CK(cudaMemsetAsync(b.slot_gain, 0, sizeof(unsigned long long) * (size_t)b.segcap, s));
  DT_CK(cudaMemsetAsync(b.slot_pos, 0xFF, sizeof(unsigned long long) * (size_t)b.segcap, s));
  // candidate pieces carry the level that wrote them; none may match before it is written
  DT_CK(cudaMemsetAsync(b.head_cand, 0xFF, sizeof(Cand2) * (size_t)b.segcap, s));
  DT_CK(cudaMemsetAsync(b.cont_cand, 0xFF, sizeof(Cand2) * (size_t)(2 * b.max_chunks), s));
  return DT_OK;
}

dt_status fit_enqueue(const FitBufs& b, const float* X, const double* y, int64_t n, int32_t d, int32_t max_depth,
                      int64_t min_leaf, cudaStream_t s, bool poll, std::vector<Pending>* pending) {
  dt_status st = clear_pieces(b, s);
  if (st != DT_OK) return st;
  DT_CK(cudaMemsetAsync(b.ctl, 0, sizeof(Ctl), s));
  {
    Nvtx range("dt presort");
    st = presort_enqueue(b, X, y, n, d, d, 0, max_depth, min_leaf, s);
  }
  if (st != DT_OK) return st;
  return fit_levels(b, d, max_depth, min_leaf, s, poll, pending);
}

// The virtual-root pass and the level loop, from the level-0 lists, root and tables.
dt_status fit_levels(const FitBufs& b, int32_t d, int32_t max_depth, int64_t min_leaf, cudaStream_t s, bool poll,
                     std::vector<Pending>* pending) {
  dt_status st;
  Ctl* ctl = b.ctl;
  // the virtual-root pass: the root's candidates and statistics
  {
    LevelArgs la{-1, 0, 0, d, min_leaf, false};
    int pr = prof_begin(PK_SCAN, s, 3);
    st = level_agg_enqueue(b, la, s);
    if (st != DT_OK) return st;
    prof_end(pr, s, 0.0);
    if (pending) pending->push_back({pr, -1, PK_SCAN});
    pr = prof_begin(PK_PARTITION, s, 2);
    st = level_fused_enqueue(b, la, s);
    if (st != DT_OK) return st;
    prof_end(pr, s, 0.0);
    if (pending) pending->push_back({pr, -1, PK_PARTITION});
  }
  const int g_sel = num_sms() * 4;
  const int g_gl = grid_of((const void*)goleft_kernel, 256, 0);
  const int g_tab = num_sms() * 4;
  for (int level = 0;; ++level) {
    char nv[32];
    snprintf(nv, sizeof nv, "dt level %d", level);
    Nvtx range(nv);
    const int par = level & 1;
    const int cur = par;  // level l lists: buffer l & 1 (the virtual-root pass writes nothing)
    // ---- piece positions + select (a5, a8)
    SelectArgs se;
    se.gbits = reinterpret_cast<uint4*>(b.gbits);
    se.nvec = b.nwords4 / 4;
    se.nodes = b.nodes[par];
    se.segs_prev = level == 0 ? b.segs[0] : b.segs[par ^ 1];
    se.ctl = ctl;
    se.par = par;
    se.level = level;
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
    se.world = 1;
    int pr = prof_begin(PK_SELECT, s, 2);
    piece_pos_kernel<<<num_sms() * 4, 256, 0, s>>>(ctl, par, d, (uint32_t)level, b.head_cand, b.cont_cand,
                                                    b.slot_gain, b.slot_pos);
    select_kernel<<<g_sel, 256, 0, s>>>(se);
    prof_end(pr, s, 0.0);
    DT_CK(cudaGetLastError());
    if (max_depth >= 0 && level == max_depth) break;
    // ---- number (a3, a8) + tables
    NumberArgs na;
    na.nodes = b.nodes[par];
    na.next = b.nodes[par ^ 1];
    na.dec = b.dec;
    na.ctl = ctl;
    na.par = par;
    na.level = level;
    na.d = d;
    na.max_depth = max_depth;
    na.min_leaf = min_leaf;
    na.out = b.dout;
    na.log = b.lvlog;
    pr = prof_begin(PK_NUMBER, s, 3);
    na.wst = b.wst;
    number_kernel<<<1, 1024, 0, s>>>(na);
    children_kernel<<<g_tab, 256, 0, s>>>(na);
    tables_kernel<<<g_tab, 256, 0, s>>>(ctl, par, d, b.nodes[par ^ 1], b.dec, b.segs[par], b.segs[par ^ 1], b.pseg, 0,
                                        b.unit_list, b.small_list);
    prof_end(pr, s, 0.0);
    DT_CK(cudaGetLastError());
    // ---- go-left bitmap (a6)
    pr = prof_begin(PK_GOLEFT, s, 1);
    goleft_kernel<<<g_gl, 256, 0, s>>>(ctl, par, b.desc[par], b.pseg, b.lr[cur], b.gbits, d);
    prof_end(pr, s, 0.0);
    if (pending) pending->push_back({pr, level, PK_GOLEFT});
    DT_CK(cudaGetLastError());
    // ---- fused partition + children's split search (a4, a7)
    LevelArgs la{level, cur, par, d, min_leaf, false};
    pr = prof_begin(PK_SCAN, s, 3);
    st = level_agg_enqueue(b, la, s);
    if (st != DT_OK) return st;
    prof_end(pr, s, 0.0);
    if (pending) pending->push_back({pr, level, PK_SCAN});
    pr = prof_begin(PK_PARTITION, s, 2);
    st = level_fused_enqueue(b, la, s);
    if (st != DT_OK) return st;
    prof_end(pr, s, 0.0);
    if (pending) pending->push_back({pr, level, PK_PARTITION});
    // unlimited depth (or a deep limit): poll the node count every few levels
    if (poll && (max_depth < 0 || max_depth > 24) && (level % 8) == 7) {
      uint32_t kk[2];
      DT_CK(cudaMemcpyAsync(kk, ctl->K, sizeof kk, cudaMemcpyDeviceToHost, s));
      DT_CK(cudaStreamSynchronize(s));
      if (kk[par ^ 1] == 0) break;
    }
  }
  return DT_OK;
}

// Reads the result back and builds the tree object (host nodes + device packed copy).
dt_status fit_finish(const FitBufs& b, int32_t d, cudaStream_t s, const std::vector<Pending>* pending,
                     dt_tree** out) {
  Ctl hc;
  DT_CK(cudaMemcpyAsync(&hc, b.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
  std::vector<LevelLog> hlog;
  if (pending && !pending->empty()) {
    hlog.resize(kMaxLogLevels);
    DT_CK(cudaMemcpyAsync(hlog.data(), b.lvlog, sizeof(LevelLog) * kMaxLogLevels, cudaMemcpyDeviceToHost, s));
  }
  DT_CK(cudaStreamSynchronize(s));
  if (pending) {
    // algorithmic bytes per launch, counted with the
    // method's f64 y:
    //   scan  (F_A + F_B): the parent level's row ids and y (4 + 8 B per entry);
    //   fused (F_C): every moved entry read and written (x 4 + row 4 + y 8 B, each way):
    //                32 B per split eval of the children (virtual-root pass: x + y read);
    //   goleft: one row id (4 B) + one bit per row.
    for (const Pending& p : *pending) {
      if (p.rec < 0 || p.level >= kMaxLogLevels) continue;
      double T = 0.0, Tn = 0.0;
      if (p.level < 0) {
        T = (double)b.n * b.d;
        Tn = T;
      } else {
        const LevelLog& L = hlog[(size_t)p.level];
        T = (double)L.T;
        Tn = (double)L.T_next;
      }
      double bytes = 0.0;
      if (p.kind == PK_SCAN) bytes = 12.0 * T;
      else if (p.kind == PK_GOLEFT) bytes = 4.125 * T / b.d;
      else if (p.kind == PK_PARTITION) bytes = (p.level < 0) ? 12.0 * T : 16.0 * T + 16.0 * Tn;
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
  t->async_alloc = 1;
  DT_CK(cudaGetDevice(&t->device));
  const bool wide = count >= kWideNodes;
  cudaError_t e = wide ? cudaMallocAsync((void**)&t->dev_wide, sizeof(uint4) * (size_t)count, s)
                       : cudaMallocAsync((void**)&t->dev_packed, sizeof(uint2) * (size_t)count, s);
  if (e == cudaSuccess) e = cudaMallocAsync((void**)&t->dev_value, sizeof(double) * (size_t)count, s);
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
  bool prof = false;               // captured with profiling event-record nodes
  std::vector<GRec> grecs;         // their events
  std::vector<Pending> pending;    // their byte counts (from the level log)
  ~FitPlan() {
    if (exec) cudaGraphExecDestroy(exec);
    prof_destroy_graph_recs(grecs);
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

void forest_graph_release();
dt_status release_workspace_impl() {
  {
    std::lock_guard<std::mutex> lk(g_plan_mu);
    for (auto& p : g_plans) p.reset();
  }
  forest_graph_release();
  DT_CK(cudaDeviceSynchronize());
  int dev = 0;
  DT_CK(cudaGetDevice(&dev));
  cudaMemPool_t pool;
  DT_CK(cudaDeviceGetDefaultMemPool(&pool, dev));
  DT_CK(cudaMemPoolTrimTo(pool, 0));
  return DT_OK;
}

// Keep freed stream-ordered workspace in the device's default pool for the next call (no
// cudaMalloc on the hot path); dt_release_workspace trims it.
dt_status keep_pool(int dev) {
  cudaMemPool_t pool;
  DT_CK(cudaDeviceGetDefaultMemPool(&pool, dev));
  uint64_t thr = UINT64_MAX;
  DT_CK(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
  return DT_OK;
}

dt_status fit_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t max_depth,
                   int64_t min_leaf, cudaStream_t s, dt_tree** out) {
  int dev = 0;
  DT_CK(cudaGetDevice(&dev));
  {
    dt_status ps = keep_pool(dev);
    if (ps != DT_OK) return ps;
  }
  static int graph_env = -1;
  if (graph_env < 0) {
    const char* e = getenv("DT_FIT_GRAPH");
    graph_env = (e && e[0] == '0') ? 0 : 1;
  }
  const bool gprof = prof_graph_mode();
  const bool use_graph = graph_env && (!prof_enabled() || gprof) && max_depth >= 0 && max_depth <= 24;
  if (use_graph) {
    std::lock_guard<std::mutex> lk(g_plan_mu);
    FitPlan* pl = nullptr;
    for (auto& p : g_plans)
      if (p && p->X == X && p->y == y && p->n == n && p->d == d && p->max_depth == max_depth &&
          p->min_leaf == min_leaf && p->device == dev && p->prof == gprof)
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
      // the workspace depends on (n, d, max_depth) and, through the node capacity, on
      // min_samples_leaf: a plan sized for a smaller m holds every larger one
      const bool same_shape = old && old->n == n && old->d == d && old->max_depth == max_depth &&
                              old->min_leaf <= min_leaf && old->device == dev;
      if (same_shape) {
        // keep the workspace, re-capture only -- no cudaFree / cudaMalloc of ~32 B per entry
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
      np->prof = gprof;
      if (!same_shape) {
        auto get = [&](auto** p, size_t count) -> cudaError_t {
          cudaError_t e = cudaMalloc((void**)p, sizeof(**p) * (count ? count : 1));
          if (e == cudaSuccess) np->mem.push_back((void*)*p);
          return e;
        };
        dt_status st = fit_alloc(np->b, n, n, d, max_depth, min_leaf, 1, get);
        if (st != DT_OK) {
          // no room beside the other cached plan(s): drop them and try once more
          bool others = false;
          for (auto& p : g_plans) others |= (bool)p;
          for (void* m : np->mem) cudaFree(m);
          np->mem.clear();
          np->b = FitBufs{};
          if (!others) return st;
          for (auto& p : g_plans) p.reset();
          st = fit_alloc(np->b, n, n, d, max_depth, min_leaf, 1, get);
          if (st != DT_OK) return st;
        }
        DT_CK(cudaStreamCreateWithFlags(&np->cap, cudaStreamNonBlocking));
      }
      const int64_t l0 = dt_launch_count();
      DT_CK(cudaStreamBeginCapture(np->cap, cudaStreamCaptureModeThreadLocal));
      if (gprof) prof_capture_target(&np->grecs);
      dt_status st = fit_enqueue(np->b, X, y, n, d, max_depth, min_leaf, np->cap, false, gprof ? &np->pending : nullptr);
      prof_capture_target(nullptr);
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
    if (!pl->prof) return fit_finish(pl->b, d, s, nullptr, out);
    // profiled replay: the byte counts from this replay's level log, then its event times
    prof_capture_target(&pl->grecs);
    dt_status fs = fit_finish(pl->b, d, s, &pl->pending, out);
    prof_capture_target(nullptr);
    if (fs == DT_OK) prof_collect_graph(pl->grecs);
    return fs;
  }
  // Direct path: stream-ordered workspace, kernels enqueued one by one.
  Workspace ws;
  ws.s = s;
  FitBufs b{};
  auto get = [&](auto** p, size_t count) -> cudaError_t { return ws.get(p, count); };
  dt_status st = fit_alloc(b, n, n, d, max_depth, min_leaf, 1, get);
  if (st != DT_OK) return st;
  std::vector<Pending> pending;
  st = fit_enqueue(b, X, y, n, d, max_depth, min_leaf, s, true, &pending);
  if (st != DT_OK) return st;
  return fit_finish(b, d, s, &pending, out);
}

// Value-range row-sharded fit: rank p holds rows
// [row_offset, row_offset + n_local) of the table; after the sharded presort it owns global
// sorted positions [p n / P, (p + 1) n / P) of every feature list and its entries never
// move between ranks again.  Per level: allgather of the per-node local bests (decided in
// rank order), OR-allreduce of the go-left bitmap, allgather of the children's boundary
// records (count, last x, S') -> rank carries of every child segment.  Every rank builds
// the same tree.  Direct enqueue; one host synchronisation per level (the node count).
namespace {
// The root's leaf rules and the virtual-root plan for another min_samples_leaf (the rest of
// the presorted state is independent of it).
__global__ void regrid_root_kernel(Ctl* ctl, NodeL* nodes0, PSeg* pseg, int d, int32_t max_depth, int64_t min_leaf) {
  const int64_t n = nodes0[0].N;
  const int srch = (max_depth != 0 && n >= 2 * min_leaf) ? 1 : 0;
  for (int f = threadIdx.x; f < d; f += blockDim.x)
    pseg[f].flags = PS_SPLIT | PS_ALLLEFT | (srch ? PS_SRCH0 : 0u);
  if (threadIdx.x == 0) {
    nodes0[0].searchable = srch;
    ctl->nsrch = (uint32_t)srch;
  }
}
}  // namespace

// (max_depth x min_samples_leaf) grid, BASELINE configs[4]: ONE presort of the table, then
// one level loop per min_samples_leaf from a snapshot of the level-0 lists and the root
// (a greedy tree depends on m only through its leaf rules; the depths
// come from truncation, dt_tree_truncate / dt_predict_eval_depths).
dt_status fit_grid_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t max_depth,
                        const int64_t* min_leafs, int32_t count, cudaStream_t s, dt_tree** outs) {
  int dev = 0;
  DT_CK(cudaGetDevice(&dev));
  {
    dt_status ps = keep_pool(dev);
    if (ps != DT_OK) return ps;
  }
  int64_t mmin = min_leafs[0];
  for (int i = 1; i < count; ++i) mmin = std::min(mmin, min_leafs[i]);
  Workspace ws;
  ws.s = s;
  FitBufs b{};
  auto get = [&](auto** p, size_t c) -> cudaError_t { return ws.get(p, c); };
  dt_status st = fit_alloc(b, n, n, d, max_depth, mmin, 1, get);
  if (st != DT_OK) return st;
  const size_t tot = (size_t)n * d;
  float* snx = nullptr;
  uint32_t* snr = nullptr;
  double* sny = nullptr;
  Ctl* snc = nullptr;
  NodeL* snn = nullptr;
  SegT* sns = nullptr;
  PSeg* snp = nullptr;
  uint32_t* snd = nullptr;
  const size_t nch0 = (tot + kChunkW - 1) / kChunkW;
  st = alloc_status(ws.get(&sns, (size_t)d));
  if (st == DT_OK) st = alloc_status(ws.get(&snp, (size_t)d));
  if (st == DT_OK) st = alloc_status(ws.get(&snd, nch0));
  if (st == DT_OK) st = alloc_status(ws.get(&snx, tot));
  if (st == DT_OK) st = alloc_status(ws.get(&snr, tot));
  if (st == DT_OK) st = alloc_status(ws.get(&sny, tot));
  if (st == DT_OK) st = alloc_status(ws.get(&snc, 1));
  if (st == DT_OK) st = alloc_status(ws.get(&snn, 1));
  if (st != DT_OK) return st;
  DT_CK(cudaMemsetAsync(b.ctl, 0, sizeof(Ctl), s));
  {
    Nvtx range("dt grid presort");
    st = presort_enqueue(b, X, y, n, d, d, 0, max_depth, min_leafs[0], s);
  }
  if (st != DT_OK) return st;
  DT_CK(cudaMemcpyAsync(snx, b.lx[0], sizeof(float) * tot, cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaMemcpyAsync(snr, b.lr[0], sizeof(uint32_t) * tot, cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaMemcpyAsync(sny, b.ly[0], sizeof(double) * tot, cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaMemcpyAsync(snc, b.ctl, sizeof(Ctl), cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaMemcpyAsync(snn, b.nodes[0], sizeof(NodeL), cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaMemcpyAsync(sns, b.segs[0], sizeof(SegT) * (size_t)d, cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaMemcpyAsync(snp, b.pseg, sizeof(PSeg) * (size_t)d, cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaMemcpyAsync(snd, b.desc[0], sizeof(uint32_t) * nch0, cudaMemcpyDeviceToDevice, s));
  for (int i = 0; i < count; ++i) {
    if (i > 0) {  // the presorted state again (the level loop consumed it)
      DT_CK(cudaMemcpyAsync(b.lx[0], snx, sizeof(float) * tot, cudaMemcpyDeviceToDevice, s));
      DT_CK(cudaMemcpyAsync(b.lr[0], snr, sizeof(uint32_t) * tot, cudaMemcpyDeviceToDevice, s));
      DT_CK(cudaMemcpyAsync(b.ly[0], sny, sizeof(double) * tot, cudaMemcpyDeviceToDevice, s));
      DT_CK(cudaMemcpyAsync(b.ctl, snc, sizeof(Ctl), cudaMemcpyDeviceToDevice, s));
      DT_CK(cudaMemcpyAsync(b.nodes[0], snn, sizeof(NodeL), cudaMemcpyDeviceToDevice, s));
      DT_CK(cudaMemcpyAsync(b.segs[0], sns, sizeof(SegT) * (size_t)d, cudaMemcpyDeviceToDevice, s));
      DT_CK(cudaMemcpyAsync(b.pseg, snp, sizeof(PSeg) * (size_t)d, cudaMemcpyDeviceToDevice, s));
      DT_CK(cudaMemcpyAsync(b.desc[0], snd, sizeof(uint32_t) * nch0, cudaMemcpyDeviceToDevice, s));
      regrid_root_kernel<<<1, 256, 0, s>>>(b.ctl, b.nodes[0], b.pseg, d, max_depth, min_leafs[i]);
      prof_add_launches(1);
      DT_CK(cudaGetLastError());
    }
    st = clear_pieces(b, s);
    if (st != DT_OK) return st;
    st = fit_levels(b, d, max_depth, min_leafs[i], s, true, nullptr);
    if (st != DT_OK) return st;
    st = fit_finish(b, d, s, nullptr, &outs[i]);
    if (st != DT_OK) return st;
  }
  return DT_OK;
}

// Random Forest: ONE presort of the table; tree t = the exact CART of
// its bootstrap sample, whose level-0 lists are the presorted lists expanded by the draw
// counts (presort.cu, forest_tree_enqueue) -- no gather, no sort per tree.
// The per-tree forest graph of the last forest on this host thread, with what it captured.
struct ForestGraph {
  FitBufs b{};
  const void* p[9] = {};
  int64_t n = 0, min_leaf = 0;
  int32_t d = 0, max_depth = 0;
  uint64_t seed = 0;
  int y32 = 0, device = -1;
  cudaGraphExec_t exec = nullptr;
  int64_t launches = 0;
  bool same(const ForestGraph& o) const {
    return memcmp(&b, &o.b, sizeof(FitBufs)) == 0 && memcmp(p, o.p, sizeof(p)) == 0 && n == o.n &&
           min_leaf == o.min_leaf && d == o.d && max_depth == o.max_depth && seed == o.seed && y32 == o.y32 &&
           device == o.device;
  }
  void reset() {
    if (exec) cudaGraphExecDestroy(exec);
    exec = nullptr;
  }
  ~ForestGraph() { reset(); }
};
thread_local ForestGraph t_forest_graph;
void forest_graph_release() { t_forest_graph.reset(); }

dt_status forest_trees_impl(const float* X, const double* y, int64_t n, int32_t d, int32_t n_trees, int32_t max_depth,
                            int64_t min_leaf, uint64_t seed, cudaStream_t s, std::vector<dt_tree*>& trees) {
  int dev = 0;
  DT_CK(cudaGetDevice(&dev));
  {
    dt_status ps = keep_pool(dev);
    if (ps != DT_OK) return ps;
  }
  Workspace ws;
  ws.s = s;
  FitBufs b{};
  auto get = [&](auto** p, size_t c) -> cudaError_t { return ws.get(p, c); };
  dt_status st = fit_alloc(b, n, n, d, max_depth, min_leaf, 1, get);
  if (st != DT_OK) return st;
  const size_t tot = (size_t)n * d;
  float* sx = nullptr;
  uint32_t *sr = nullptr, *w = nullptr;
  double *sy = nullptr, *ys = nullptr;
  unsigned long long* tsum = nullptr;
  st = alloc_status(ws.get(&sx, tot));
  if (st == DT_OK) st = alloc_status(ws.get(&sr, tot));
  if (st == DT_OK) st = alloc_status(ws.get(&sy, tot));
  if (st == DT_OK) st = alloc_status(ws.get(&w, (size_t)n));
  if (st == DT_OK) st = alloc_status(ws.get(&ys, (size_t)n));
  if (st == DT_OK) st = alloc_status(ws.get(&tsum, tot / 2048 + 2));
  if (st != DT_OK) return st;
  DT_CK(cudaMemsetAsync(b.ctl, 0, sizeof(Ctl), s));
  {
    Nvtx range("dt forest presort");
    st = presort_enqueue(b, X, y, n, d, d, 0, max_depth, min_leaf, s);
  }
  if (st != DT_OK) return st;
  Ctl hc;
  DT_CK(cudaMemcpyAsync(&hc, b.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
  DT_CK(cudaMemcpyAsync(sx, b.lx[0], sizeof(float) * tot, cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaMemcpyAsync(sr, b.lr[0], sizeof(uint32_t) * tot, cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaMemcpyAsync(sy, b.ly[0], sizeof(double) * tot, cudaMemcpyDeviceToDevice, s));
  DT_CK(cudaStreamSynchronize(s));
  if (hc.nonfinite) return fail(DT_ERR_NONFINITE, "dt_forest_fit: non-finite value in X or y");
  uint32_t* tdev = nullptr;
  st = alloc_status(ws.get(&tdev, 1));
  if (st != DT_OK) return st;
  // Bounded depth: one tree's sequence (pieces cleared, bootstrap expansion, level loop) is
  // captured once as a CUDA graph and replayed per tree with the tree index set on the
  // device.  The instantiated graph is kept (per host thread) and reused by the next forest
  // whose buffers (stream-ordered pool: usually the same addresses) and shape match.
  const bool use_graph = !prof_enabled() && max_depth >= 0 && max_depth <= 24;
  ForestGraph& fg = t_forest_graph;
  ForestGraph key;
  key.b = b;
  key.p[0] = X; key.p[1] = y; key.p[2] = sx; key.p[3] = sr; key.p[4] = sy; key.p[5] = w; key.p[6] = ys;
  key.p[7] = tsum; key.p[8] = tdev;
  key.n = n; key.d = d; key.max_depth = max_depth; key.min_leaf = min_leaf; key.seed = seed; key.y32 = hc.y32;
  DT_CK(cudaGetDevice(&key.device));
  if (use_graph && !(fg.exec && fg.same(key))) {
    fg.reset();
    cudaStream_t cap = nullptr;
    DT_CK(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
    struct DropStream {
      cudaStream_t c;
      ~DropStream() { cudaStreamDestroy(c); }
    } drop_cap{cap};
    const int64_t l0 = dt_launch_count();
    DT_CK(cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal));
    st = clear_pieces(b, cap);
    if (st == DT_OK)
      st = forest_tree_enqueue(b, sx, sr, sy, y, n, d, max_depth, min_leaf, seed, tdev, hc.y32, w, ys, tsum, cap);
    if (st == DT_OK) st = fit_levels(b, d, max_depth, min_leaf, cap, false, nullptr);
    cudaGraph_t graph = nullptr;
    const cudaError_t ce = cudaStreamEndCapture(cap, &graph);
    if (st != DT_OK) {
      if (graph) cudaGraphDestroy(graph);
      return st;
    }
    if (ce != cudaSuccess) return cuda_fail(ce, "cudaStreamEndCapture", __FILE__, __LINE__);
    const int64_t per_tree = dt_launch_count() - l0;
    prof_add_launches(-per_tree);  // counted per replay
    cudaGraphExec_t exec = nullptr;
    const cudaError_t ie = cudaGraphInstantiate(&exec, graph, 0);
    cudaGraphDestroy(graph);
    if (ie != cudaSuccess) return cuda_fail(ie, "cudaGraphInstantiate", __FILE__, __LINE__);
    key.exec = exec;
    key.launches = per_tree;
    fg = key;
    key.exec = nullptr;  // owned by the cache now
  }
  for (int32_t t = 0; t < n_trees; ++t) {
    set_u32_kernel<<<1, 1, 0, s>>>(tdev, (uint32_t)t);
    prof_add_launches(1);
    DT_CK(cudaGetLastError());
    if (use_graph) {
      DT_CK(cudaGraphLaunch(fg.exec, s));
      prof_add_launches(fg.launches);
    } else {
      st = clear_pieces(b, s);
      if (st == DT_OK)
        st = forest_tree_enqueue(b, sx, sr, sy, y, n, d, max_depth, min_leaf, seed, tdev, hc.y32, w, ys, tsum, s);
      if (st == DT_OK) st = fit_levels(b, d, max_depth, min_leaf, s, true, nullptr);
      if (st != DT_OK) return st;
    }
    dt_tree* tr = nullptr;
    st = fit_finish(b, d, s, nullptr, &tr);
    if (st != DT_OK) return st;
    trees.push_back(tr);
  }
  return DT_OK;
}

dt_status fit_sharded_impl(dt_comm* comm, const float* X, const double* y, int64_t n_local, int64_t row_offset,
                           int64_t n_global, int32_t d, int32_t max_depth, int64_t min_leaf, cudaStream_t s,
                           dt_tree** out) {
  const int P = comm_world(comm), rank = comm_rank(comm);
  int dev = 0;
  DT_CK(cudaGetDevice(&dev));
  {
    dt_status ps = keep_pool(dev);
    if (ps != DT_OK) return ps;
  }
  const int64_t nlist = std::max<int64_t>(std::max<int64_t>(n_local, (n_global + P - 1) / P), 1);
  Workspace ws;
  ws.s = s;
  FitBufs b{};
  auto get = [&](auto** p, size_t count) -> cudaError_t { return ws.get(p, count); };
  dt_status st = fit_alloc(b, nlist, n_global, d, max_depth, min_leaf, std::max(P, 2), get);
  if (st != DT_OK) return st;
  std::vector<Pending> pending;
  DT_CK(cudaMemsetAsync(b.slot_gain, 0, sizeof(unsigned long long) * (size_t)b.segcap, s));
  DT_CK(cudaMemsetAsync(b.slot_pos, 0xFF, sizeof(unsigned long long) * (size_t)b.segcap, s));
  DT_CK(cudaMemsetAsync(b.head_cand, 0xFF, sizeof(Cand2) * (size_t)b.segcap, s));
  DT_CK(cudaMemsetAsync(b.cont_cand, 0xFF, sizeof(Cand2) * (size_t)(2 * b.max_chunks), s));
  DT_CK(cudaMemsetAsync(b.ctl, 0, sizeof(Ctl), s));
  {
    Nvtx range("dt sharded presort");
    st = presort_sharded_enqueue(b, comm, X, y, n_local, row_offset, n_global, d, max_depth, min_leaf, s);
  }
  if (st != DT_OK) return st;
  Ctl* ctl = b.ctl;
  {  // the virtual-root pass (the root's rank carries come from the presort)
    LevelArgs la{-1, 0, 0, d, min_leaf, false};
    int pr = prof_begin(PK_SCAN, s, 3);
    pending.push_back({pr, -1, PK_SCAN});
    st = level_agg_enqueue(b, la, s);
    if (st != DT_OK) return st;
    prof_end(pr, s, 0.0);
    pr = prof_begin(PK_PARTITION, s, 2);
    pending.push_back({pr, -1, PK_PARTITION});
    st = level_fused_enqueue(b, la, s);
    if (st != DT_OK) return st;
    prof_end(pr, s, 0.0);
  }
  const int g_sel = num_sms() * 4;
  const int g_gl = grid_of((const void*)goleft_kernel, 256, 0);
  const int g_tab = num_sms() * 4;
  uint32_t K = 1;  // nodes at the level (host copy)
  for (int level = 0;; ++level) {
    char nv[32];
    snprintf(nv, sizeof nv, "dt sharded level %d", level);
    Nvtx range(nv);
    const int par = level & 1, cur = par;
    SelectArgs se;
    se.gbits = reinterpret_cast<uint4*>(b.gbits);
    se.nvec = b.nwords4 / 4;
    se.nodes = b.nodes[par];
    se.segs_prev = level == 0 ? b.segs[0] : b.segs[par ^ 1];
    se.ctl = ctl;
    se.par = par;
    se.level = level;
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
    se.world = P;
    int pr = prof_begin(PK_SELECT, s, 3);
    piece_pos_kernel<<<num_sms() * 4, 256, 0, s>>>(ctl, par, d, (uint32_t)level, b.head_cand, b.cont_cand,
                                                    b.slot_gain, b.slot_pos);
    select_kernel<<<g_sel, 256, 0, s>>>(se);
    DT_CK(cudaGetLastError());
    st = comm_allgather(comm, b.exch_send, b.exch_all, sizeof(ExchRec) * (size_t)K, s);
    if (st != DT_OK) return st;
    decide_kernel<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>((K + 255) / 256, num_sms() * 4)), 256, 0, s>>>(
        se, b.exch_all, (int64_t)K);
    prof_end(pr, s, 0.0);
    DT_CK(cudaGetLastError());
    if (max_depth >= 0 && level == max_depth) break;
    NumberArgs na;
    na.nodes = b.nodes[par];
    na.next = b.nodes[par ^ 1];
    na.dec = b.dec;
    na.ctl = ctl;
    na.par = par;
    na.level = level;
    na.d = d;
    na.max_depth = max_depth;
    na.min_leaf = min_leaf;
    na.out = b.dout;
    na.log = b.lvlog;
    pr = prof_begin(PK_NUMBER, s, 2);
    na.wst = b.wst;
    number_kernel<<<1, 1024, 0, s>>>(na);
    children_kernel<<<g_tab, 256, 0, s>>>(na);
    prof_end(pr, s, 0.0);
    DT_CK(cudaGetLastError());
    uint32_t hk[2], hsrch = 0;
    DT_CK(cudaMemcpyAsync(hk, ctl->K, sizeof hk, cudaMemcpyDeviceToHost, s));
    DT_CK(cudaMemcpyAsync(&hsrch, &ctl->nsrch, sizeof hsrch, cudaMemcpyDeviceToHost, s));
    DT_CK(cudaStreamSynchronize(s));
    const uint32_t K2 = hk[par ^ 1];
    if (K2 == 0) break;  // every node of the level is a leaf (same on every rank)
    // plans of the level's segments (their go-left counts feed the bitmap)
    tables_kernel<<<g_tab, 256, 0, s>>>(ctl, par, d, b.nodes[par ^ 1], b.dec, b.segs[par], b.segs[par ^ 1], b.pseg, 1,
                                        b.unit_list, b.small_list);
    DT_CK(cudaGetLastError());
    // go-left bitmap: each rank sets the bits of its own split-feature entries; OR over ranks
    pr = prof_begin(PK_GOLEFT, s, 1);
    pending.push_back({pr, level, PK_GOLEFT});
    goleft_kernel<<<g_gl, 256, 0, s>>>(ctl, par, b.desc[par], b.pseg, b.lr[cur], b.gbits, d);
    DT_CK(cudaGetLastError());
    st = comm_allreduce_or_u32(comm, b.gbits, b.nwords4, s);
    if (st != DT_OK) return st;
    prof_end(pr, s, 0.0);
    LevelArgs la{level, cur, par, d, min_leaf, true};
    pr = prof_begin(PK_SCAN, s, 3);
    pending.push_back({pr, level, PK_SCAN});
    st = level_agg_enqueue(b, la, s);
    if (st != DT_OK) return st;
    prof_end(pr, s, 0.0);
    if (hsrch > 0) {
      // children's boundary records -> their segments (positions, rank carries)
      const int64_t n2 = (int64_t)K2 * d;
      bnd_kernel<<<g_tab, 256, 0, s>>>(ctl, par, d, b.pseg, b.tails, b.cexcl, b.bcarry, b.bnd_send);
      DT_CK(cudaGetLastError());
      st = comm_allgather(comm, b.bnd_send, b.bnd_all, sizeof(BndRec) * (size_t)n2, s);
      if (st != DT_OK) return st;
      unsigned long long* excl = b.scan_tmp;
      unsigned long long* btot = b.scan_tmp + b.segcap;
      segscan_kernel<<<(unsigned)((n2 + 1023) / 1024), 1024, 0, s>>>(ctl, par, d, b.nodes[par ^ 1], b.bnd_send,
                                                                      excl, btot);
      segwrite_kernel<<<g_tab, 256, 0, s>>>(ctl, par, d, rank, b.nodes[par ^ 1], b.bnd_all, excl, btot,
                                            b.segs[par ^ 1]);
      tables_kernel<<<g_tab, 256, 0, s>>>(ctl, par, d, b.nodes[par ^ 1], b.dec, b.segs[par], b.segs[par ^ 1], b.pseg,
                                          2, b.unit_list, b.small_list);
      DT_CK(cudaGetLastError());
    } else {
      // no searchable child: statistics only, nothing is written (empty next lists)
      DT_CK(cudaMemsetAsync(&ctl->T[par ^ 1], 0, sizeof(unsigned long long), s));
      DT_CK(cudaMemsetAsync(&ctl->T0[par ^ 1], 0, sizeof(unsigned long long), s));
    }
    pr = prof_begin(PK_PARTITION, s, 2);
    pending.push_back({pr, level, PK_PARTITION});
    st = level_fused_enqueue(b, la, s);
    if (st != DT_OK) return st;
    prof_end(pr, s, 0.0);
    K = K2;
  }
  return fit_finish(b, d, s, &pending, out);
}

}  // namespace dtl
