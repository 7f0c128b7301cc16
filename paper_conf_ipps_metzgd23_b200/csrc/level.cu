// The fused per-level pass of the exact CART fit:
// stable partition of the level-l feature lists into the children's level-(l+1) lists
// AND evaluation of every split candidate of every child (every feature, every
// threshold), in one pass over the entries.
//
//   F_A  level_agg_kernel   per warp chunk (256 entries): go-left bit of every entry
//                           (bitmap lookup by row id), and the chunk aggregate AggP
//                           (left count, child-centred sums of both sides, last x of
//                           both sides) since the chunk's last segment head;
//   F_B  agg_scan_kernel    fixed-shape exclusive scan of the chunk aggregates -> the
//                           carry of every chunk (blocks of kBlockChunks chunks + block carries);
//   F_C  fused_kernel       per warp chunk, a TMA bulk-copy pipeline (x, row, y, bits,
//                           segment plan, carries): the chunk's entries are written to
//                           their child lists (stable: left entries in order, then right
//                           entries in order) with coalesced row-wise stores, and the
//                           children's prefix sums S'_L, positions and neighbour x give
//                           the exact gain of every valid position (compacted, one gain
//                           per valid position); per (child segment, chunk) the best
//                           candidate is recorded, per child node the statistics
//                           (sum (y - v)^2, min, max, sum (y - c)) from feature 0.
// All sums run in a fixed order (within a lane sequentially, across lanes Kogge-Stone,
// across chunks the F_B tree), so results are bit-reproducible; in integer mode every
// sum is exact, so the trees are independent of the summation order (Reading R17).
#include <algorithm>
#include <type_traits>

#include "bulk.cuh"
#include "fit_core.cuh"

namespace dtl {

namespace {

constexpr int kThreads = 256;
#ifndef DT_FUSED_THREADS
#define DT_FUSED_THREADS 256  // threads per CTA of the fused pass (per-warp work: no block barriers)
#endif
constexpr int kFusedThreads = DT_FUSED_THREADS;
#ifndef DT_FUSED_STAGES
#define DT_FUSED_STAGES 2  // bulk-copy stages per warp of the fused pass (3 measured: no faster)
#endif
constexpr int kStages = DT_FUSED_STAGES;
#ifndef DT_FUSED_MINB
#define DT_FUSED_MINB 2  // CTAs per SM of the fused pass (register budget; 3 spills: slower)
#endif
constexpr float kNaN = __builtin_nanf("");
// chunk aggregate x fields: a NaN with this payload | item index = "x of entry index of
// this chunk" (resolved by agg_scan_kernel); the plain NaN means "none" (x is finite)
constexpr uint32_t kXMark = 0x7FE00000u;

__device__ __forceinline__ double y_at(const double* __restrict__ ly, int64_t p, bool y32) {
  return y32 ? (double)reinterpret_cast<const int32_t*>(ly)[p] : ly[p];
}

// ----------------------------------------------------------------------------- F_A --

struct AggArgs {
  bool walk_gen;  // general chunks by the per-item segment walk (virtual root, sharded tails)
  const uint32_t* lr;
  const double* ly;
  const float* lx;
  const uint32_t* desc;
  const PSeg* pseg;
  const uint32_t* gbits;
  uint8_t* gm;
  AggP* agg;
  AggP* tails;
  const uint2* fast_list;
  const uint32_t* gen_list;
  const Ctl* ctl;
  int par;
  uint32_t d;  // lists per level (segments of the parent level: K * d)
  int64_t nwords;
};

__device__ __forceinline__ void load_rows_y(const AggArgs& a, int64_t p0, int64_t T, bool y32, bool need_rows,
                                            uint32_t* rv, double* yv) {
  if (p0 + kItems <= T) {
    if (need_rows) {
      const uint4* r4 = reinterpret_cast<const uint4*>(a.lr + p0);
      const uint4 q0 = __ldcs(r4), q1 = __ldcs(r4 + 1);
      rv[0] = q0.x; rv[1] = q0.y; rv[2] = q0.z; rv[3] = q0.w;
      rv[4] = q1.x; rv[5] = q1.y; rv[6] = q1.z; rv[7] = q1.w;
    }
    if (y32) {
      const int4* y4 = reinterpret_cast<const int4*>(reinterpret_cast<const int32_t*>(a.ly) + p0);
      const int4 q0 = __ldcs(y4), q1 = __ldcs(y4 + 1);
      yv[0] = q0.x; yv[1] = q0.y; yv[2] = q0.z; yv[3] = q0.w;
      yv[4] = q1.x; yv[5] = q1.y; yv[6] = q1.z; yv[7] = q1.w;
    } else {
      const double2* y2 = reinterpret_cast<const double2*>(a.ly + p0);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const double2 t = __ldcs(y2 + q);
        yv[2 * q] = t.x;
        yv[2 * q + 1] = t.y;
      }
    }
  } else {
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
      const bool ok = p0 + j < T;
      rv[j] = (ok && need_rows) ? a.lr[p0 + j] : 0u;
      yv[j] = ok ? y_at(a.ly, p0 + j, y32) : 0.0;
    }
  }
}

// Kogge-Stone inclusive scan of two f64 values across the warp (fixed shape).
__device__ __forceinline__ void warp_incl2(double& a, double& b) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const double oa = __shfl_up_sync(0xffffffffu, a, d);
    const double ob = __shfl_up_sync(0xffffffffu, b, d);
    if (lane >= d) {
      a = __dadd_rn(oa, a);
      b = __dadd_rn(ob, b);
    }
  }
}

template <class T>
__device__ __forceinline__ T warp_excl_seg(T v, const T& ident, T& agg) {
  const int lane = threadIdx.x & 31;
  T inc = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    T o = shfl_up(inc, d);
    if (lane >= d) inc = combine(o, inc);
  }
  agg = shfl_idx(inc, 31);
  T ex = shfl_up(inc, 1);
  if (lane == 0) ex = ident;
  return ex;
}

// Segment plan fields the aggregate pass needs.
struct SegLite {
  uint64_t start, end;
  uint32_t flags;
  double c0, c1;
};
__device__ __forceinline__ SegLite seg_lite(const PSeg* __restrict__ ps, uint32_t s) {
  SegLite r;
  r.start = __ldg(&ps[s].start);
  r.end = r.start + __ldg(&ps[s].cnt);
  r.flags = __ldg(&ps[s].flags);
  r.c0 = __ldg(&ps[s].c[0]);
  r.c1 = __ldg(&ps[s].c[1]);
  return r;
}

// Chunk plan of a pass (thread per chunk).  A chunk inside ONE segment: of a split node
// -> fast list {chunk, segment} (F_A fast path) and unit list (F_C); of a node that does
// not split -> nothing to do (its aggregate is written here).  A chunk with segment heads
// inside -> gen list (F_A general path) and, per split segment piece of more than
// kSmallSeg entries, the unit list (F_C processes the chunk once per piece, masked to the
// piece's entries).  Split segments of at most kSmallSeg entries go to the small list
// (fused_small_kernel: a warp per segment, lane = entry), from the chunk holding their
// head.  (Levels >= 0: tables_kernel lists the pieces and small segments from the segment
// side, emit_pieces; this walk serves the virtual-root pass.)  So a chunk has at most kMaxPieces pieces: k segments of >= 33 entries meeting
// 256 consecutive entries have their k - 2 middle ones inside, (k - 2) * 33 <= 254, k <= 9.
// Block-aggregated appends.
constexpr int kMaxPieces = 9;

// Block-aggregated appends to four list counters (one atomic per counter per block;
// block-uniform call: contains barriers).  pos[i] = this thread's first slot.
__device__ __forceinline__ void block_append4(const uint32_t (&cnt)[4], uint32_t* const (&ctr)[4],
                                              uint32_t (&pos)[4]) {
  __shared__ uint32_t sw[32][4];
  __shared__ uint32_t sb[4];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t inc[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    inc[i] = cnt[i];
#pragma unroll
    for (int dd = 1; dd < 32; dd <<= 1) {
      const uint32_t o = __shfl_up_sync(0xffffffffu, inc[i], dd);
      if (lane >= dd) inc[i] += o;
    }
    if (lane == 31) sw[w][i] = inc[i];
  }
  __syncthreads();
  if (threadIdx.x < 4) {
    const int i = threadIdx.x;
    uint32_t run = 0u;
    for (int q = 0; q < (int)(blockDim.x >> 5); ++q) {
      const uint32_t t = sw[q][i];
      sw[q][i] = run;
      run += t;
    }
    sb[i] = run ? atomicAdd(ctr[i], run) : 0u;
  }
  __syncthreads();
#pragma unroll
  for (int i = 0; i < 4; ++i) pos[i] = sb[i] + sw[w][i] + inc[i] - cnt[i];
  __syncthreads();  // sw / sb are reused by the next call
}

__global__ void __launch_bounds__(256) chunk_plan_kernel(Ctl* ctl, int par, int d, const uint32_t* __restrict__ desc,
                                                         const PSeg* __restrict__ pseg, AggP* __restrict__ agg,
                                                         uint2* __restrict__ fast_list, uint32_t* __restrict__ gen_list,
                                                         uint2* __restrict__ unit_list, uint32_t* __restrict__ small_list,
                                                         bool walk) {
  const uint64_t T = ctl->T[par];
  const bool full = ctl->nsrch > 0;  // children searched: every list; else feature 0 (statistics)
  const uint64_t Tw = full ? T : ctl->T0[par];
  const int64_t nch = (int64_t)((Tw + kChunkW - 1) / kChunkW);
  const uint32_t nseg = ctl->K[par] * (uint32_t)d;  // segments of the parent level
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < nch; base += stride) {  // block-uniform trip count
    const int64_t ch = base + threadIdx.x;
    bool fast = false, gen = false;
    uint32_t npieces = 0, nsmall = 0;
    uint32_t s = 0;
    const uint64_t cbase = (uint64_t)ch * kChunkW, cend = min(cbase + kChunkW, T);
    if (ch < nch) {
      s = __ldg(desc + ch);
      const uint64_t st = __ldg(&pseg[s].start), en = st + __ldg(&pseg[s].cnt);
      const bool split = (__ldg(&pseg[s].flags) & PS_SPLIT) != 0;
      if (st <= cbase && en >= cbase + kChunkW) {
        if (split) fast = true;
        else {
          AggP z = agg_ident();
          z.flag = st == cbase ? 1u : 0u;
          agg[ch] = z;
        }
      } else {
        gen = true;
        // split segments meeting this chunk (non-empty segments; empty runs skipped)
        for (uint32_t t = s; walk;) {
          const uint64_t ts = __ldg(&pseg[t].start);
          const uint32_t tc = __ldg(&pseg[t].cnt);
          if (tc && (__ldg(&pseg[t].flags) & PS_SPLIT)) {
            if (tc > kSmallSeg) ++npieces;
            else if (ts >= cbase) ++nsmall;
          }
          if (ts + tc >= cend || t + 1u >= nseg) break;
          t = seg_gallop(pseg, t + 1u, nseg - 1u, ts + tc);
        }
      }
    }
    const uint32_t cnt[4] = {fast ? 1u : 0u, gen ? 1u : 0u, nsmall, fast ? 1u : npieces};
    uint32_t* const ctr[4] = {&ctl->nfast, &ctl->ngen, &ctl->nsmall, &ctl->nunit};
    uint32_t pos[4];
    block_append4(cnt, ctr, pos);
    if (fast) {
      fast_list[pos[0]] = make_uint2((uint32_t)ch, s);
      unit_list[pos[3]] = make_uint2((uint32_t)ch, s);
    }
    if (gen) gen_list[pos[1]] = (uint32_t)ch;
    if (npieces || nsmall) {
      uint32_t pu = pos[3], psm = pos[2];
      for (uint32_t t = s;;) {
        const uint64_t ts = __ldg(&pseg[t].start);
        const uint32_t tc = __ldg(&pseg[t].cnt);
        if (tc && (__ldg(&pseg[t].flags) & PS_SPLIT)) {
          if (tc > kSmallSeg) unit_list[pu++] = make_uint2((uint32_t)ch, t);
          else if (ts >= cbase) small_list[psm++] = t;
        }
        if (ts + tc >= cend || t + 1u >= nseg) break;
        t = seg_gallop(pseg, t + 1u, nseg - 1u, ts + tc);
      }
    }
  }
}

// One fast chunk of the aggregate pass: go-left bits, sums, last x of both sides.
template <bool kSmemBits, bool kTails>
__device__ __forceinline__ void agg_fast_chunk(const AggArgs& a, const uint32_t* __restrict__ bits, int64_t ch,
                                               uint32_t s, const uint32_t* rv, const double* yv) {
  const int lane = threadIdx.x & 31;
  const uint64_t cbase = (uint64_t)ch * kChunkW;
  const int64_t p0 = (int64_t)cbase + lane * kItems;
  const uint64_t st = __ldg(&a.pseg[s].start);
  const uint32_t flags = __ldg(&a.pseg[s].flags);
  const double c0 = __ldg(&a.pseg[s].c[0]), c1 = __ldg(&a.pseg[s].c[1]);
  uint32_t gbyte = 0xffu;
  if (!(flags & PS_ALLLEFT)) {
    uint32_t wv[kItems];
#pragma unroll
    for (int j = 0; j < kItems; ++j) wv[j] = bits[rv[j] >> 5];  // independent shared-memory loads
    gbyte = 0u;
#pragma unroll
    for (int j = 0; j < kItems; ++j) gbyte |= ((wv[j] >> (rv[j] & 31)) & 1u) << j;
  }
  double sl = 0.0, sr = 0.0;
#pragma unroll
  for (int j = 0; j < kItems; ++j) {
    const bool g = (gbyte >> j) & 1u;
    const double d = __dsub_rn(yv[j], g ? c0 : c1);
    // adding +0.0 is exact: a sum of (y - c) terms is never -0.0
    sl = __dadd_rn(sl, g ? d : 0.0);
    sr = __dadd_rn(sr, g ? 0.0 : d);
  }
  warp_incl2(sl, sr);
  const uint32_t Lm = __ballot_sync(0xffffffffu, gbyte != 0u);
  const uint32_t Rm = __ballot_sync(0xffffffffu, gbyte != 0xffu);
  AggP out;
  out.flag = st == cbase ? 1u : 0u;
  out.nl = __reduce_add_sync(0xffffffffu, (uint32_t)__popc(gbyte));
  out.sl = __shfl_sync(0xffffffffu, sl, 31);
  out.sr = __shfl_sync(0xffffffffu, sr, 31);
  out.xl = kNaN;
  out.xr = kNaN;
  if (kTails) {  // sharded: the tails need the x values here
    if (Lm) {
      const int h = 31 - __clz(Lm);
      float v = 0.f;
      if (lane == h) v = a.lx[p0 + 31 - __clz(gbyte)];
      out.xl = __shfl_sync(0xffffffffu, v, h);
    }
    if (Rm) {
      const int h = 31 - __clz(Rm);
      float v = 0.f;
      if (lane == h) v = a.lx[p0 + 31 - __clz(~gbyte & 0xffu)];
      out.xr = __shfl_sync(0xffffffffu, v, h);
    }
  } else {
    // the last left / right entry's index in the chunk, as a marker NaN that agg_scan
    // resolves to its x when it loads the aggregate (no dependent x load here)
    if (Lm) {
      const int h = 31 - __clz(Lm);
      const uint32_t gh = __shfl_sync(0xffffffffu, gbyte, h);
      out.xl = __uint_as_float(kXMark | (uint32_t)(8 * h + 31 - __clz(gh)));
    }
    if (Rm) {
      const int h = 31 - __clz(Rm);
      const uint32_t gh = __shfl_sync(0xffffffffu, gbyte, h);
      out.xr = __uint_as_float(kXMark | (uint32_t)(8 * h + 31 - __clz(~gh & 0xffu)));
    }
  }
  a.gm[cbase / 8 + lane] = (uint8_t)gbyte;
  if (lane == 0) {
    a.agg[ch] = out;
    if (kTails && st + __ldg(&a.pseg[s].cnt) == cbase + kChunkW) a.tails[s] = out;
  }
}

template <bool kSmemBits, bool kTails>
__global__ void __launch_bounds__(kSmemBits ? 1024 : kThreads) level_agg_kernel(AggArgs a) {
  extern __shared__ uint4 smem_bits4[];
  const uint32_t* __restrict__ bits = kSmemBits ? reinterpret_cast<const uint32_t*>(smem_bits4) : a.gbits;
  const uint64_t T = a.ctl->T[a.par];
  const bool y32 = a.ctl->y32 != 0;
  const int64_t nfast = a.ctl->nfast, ngen = a.ctl->ngen;
  // the go-left bitmap into shared memory by bulk copies (TMA), completed on an mbarrier:
  // the first chunk's rows and y are fetched while it lands
  __shared__ uint64_t sbar;
  if (kSmemBits) {
    if (threadIdx.x == 0) {
      mbar_init(&sbar, 1);
      mbar_init_fence();
      const uint32_t bytes = (uint32_t)(a.nwords * 4);
      mbar_arrive_expect_tx(&sbar, bytes);
      constexpr uint32_t kPiece = 32768u;
      for (uint32_t o = 0; o < bytes; o += kPiece)
        bulk_g2s(reinterpret_cast<unsigned char*>(smem_bits4) + o, reinterpret_cast<const unsigned char*>(a.gbits) + o,
                 min(kPiece, bytes - o), &sbar);
    }
    __syncthreads();  // the barrier is initialised before anyone waits on it
  }
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  // ---- fast chunks: the next chunk's rows and y are in flight during this chunk
  if (y32) {
    uint2 e = gw < nfast ? a.fast_list[gw] : make_uint2(0u, 0u);
    uint4 r0 = make_uint4(0, 0, 0, 0), r1 = r0;
    int4 q0 = make_int4(0, 0, 0, 0), q1 = q0;
    auto fetch = [&](const uint2& en) {
      const int64_t p0 = (int64_t)en.x * kChunkW + lane * kItems;
      const uint4* r4 = reinterpret_cast<const uint4*>(a.lr + p0);
      const int4* y4 = reinterpret_cast<const int4*>(reinterpret_cast<const int32_t*>(a.ly) + p0);
      r0 = __ldcs(r4); r1 = __ldcs(r4 + 1);
      q0 = __ldcs(y4); q1 = __ldcs(y4 + 1);
    };
    if (gw < nfast) fetch(e);
    if (kSmemBits) mbar_wait(&sbar, 0);
    for (int64_t i = gw; i < nfast; i += nw) {
      const uint2 cur = e;
      const uint32_t rv[kItems] = {r0.x, r0.y, r0.z, r0.w, r1.x, r1.y, r1.z, r1.w};
      const double yv[kItems] = {(double)q0.x, (double)q0.y, (double)q0.z, (double)q0.w,
                                 (double)q1.x, (double)q1.y, (double)q1.z, (double)q1.w};
      if (i + nw < nfast) {
        e = a.fast_list[i + nw];
        fetch(e);
      }
      agg_fast_chunk<kSmemBits, kTails>(a, bits, (int64_t)cur.x, cur.y, rv, yv);
    }
  } else {
    if (kSmemBits) mbar_wait(&sbar, 0);
    for (int64_t i = gw; i < nfast; i += nw) {
      const uint2 cur = a.fast_list[i];
      uint32_t rv[kItems];
      double yv[kItems];
      load_rows_y(a, (int64_t)cur.x * kChunkW + lane * kItems, (int64_t)T, false, true, rv, yv);
      agg_fast_chunk<kSmemBits, kTails>(a, bits, (int64_t)cur.x, cur.y, rv, yv);
    }
  }
  // ---- general chunks: segment heads inside; per item walk
  if (kSmemBits) mbar_wait(&sbar, 0);
  const uint32_t nseg = a.ctl->K[a.par] * a.d;
  if (!kTails && !a.walk_gen) {
    // The chunk's aggregate only needs its LAST segment's entries (the scan restarts at
    // that segment's head): one segment lookup per chunk, no per-item walk.  The go-left
    // bits of every entry (F_C's pieces of the other segments read them) are looked up
    // regardless of the segment (levels >= 0 have no all-left segments).
    for (int64_t gi = gw; gi < ngen; gi += nw) {
      const int64_t ch = (int64_t)a.gen_list[gi];
      const uint64_t cbase = (uint64_t)ch * kChunkW;
      const int64_t p0 = (int64_t)cbase + lane * kItems;
      const uint64_t plast = min(cbase + (uint64_t)kChunkW, T) - 1u;
      uint32_t sidx = __ldg(a.desc + ch);
      SegLite g = seg_lite(a.pseg, sidx);
      if (plast >= g.end) {
        sidx = seg_gallop(a.pseg, sidx + 1u, nseg - 1u, plast);
        g = seg_lite(a.pseg, sidx);
      }
      uint32_t rv[kItems];
      double yv[kItems];
      load_rows_y(a, p0, (int64_t)T, y32, true, rv, yv);
      uint32_t gbyte = 0u, inl = 0u;  // go-left bits; my items in the last segment (and split)
      const bool split = (g.flags & PS_SPLIT) != 0;
#pragma unroll
      for (int j = 0; j < kItems; ++j) {
        const uint64_t p = (uint64_t)p0 + j;
        if (p < T) {
          gbyte |= ((bits[rv[j] >> 5] >> (rv[j] & 31)) & 1u) << j;
          if (split && p >= g.start) inl |= 1u << j;
        }
      }
      double sl = 0.0, sr = 0.0;
#pragma unroll
      for (int j = 0; j < kItems; ++j) {
        const bool in = (inl >> j) & 1u, gl = (gbyte >> j) & 1u;
        const double dd = __dsub_rn(yv[j], gl ? g.c0 : g.c1);
        // adding +0.0 is exact: a sum of (y - c) terms is never -0.0
        sl = __dadd_rn(sl, in && gl ? dd : 0.0);
        sr = __dadd_rn(sr, in && !gl ? dd : 0.0);
      }
      warp_incl2(sl, sr);
      const uint32_t lb = gbyte & inl, rb = ~gbyte & inl;
      const uint32_t Lm = __ballot_sync(0xffffffffu, lb != 0u);
      const uint32_t Rm = __ballot_sync(0xffffffffu, rb != 0u);
      AggP out = agg_ident();
      out.flag = g.start >= cbase ? 1u : 0u;
      out.nl = __reduce_add_sync(0xffffffffu, (uint32_t)__popc(lb));
      out.sl = __shfl_sync(0xffffffffu, sl, 31);
      out.sr = __shfl_sync(0xffffffffu, sr, 31);
      if (Lm) {
        const int h = 31 - __clz(Lm);
        const uint32_t gh = __shfl_sync(0xffffffffu, lb, h);
        out.xl = __uint_as_float(kXMark | (uint32_t)(8 * h + 31 - __clz(gh)));
      }
      if (Rm) {
        const int h = 31 - __clz(Rm);
        const uint32_t gh = __shfl_sync(0xffffffffu, rb, h);
        out.xr = __uint_as_float(kXMark | (uint32_t)(8 * h + 31 - __clz(gh)));
      }
      a.gm[cbase / 8 + lane] = (uint8_t)gbyte;
      if (lane == 0) a.agg[ch] = out;
    }
    return;
  }
  for (int64_t gi = gw; gi < ngen; gi += nw) {
    const int64_t ch = (int64_t)a.gen_list[gi];
    const uint64_t cbase = (uint64_t)ch * kChunkW;
    const int64_t p0 = (int64_t)cbase + lane * kItems;
    const uint32_t s = __ldg(a.desc + ch);
    const SegLite sg = seg_lite(a.pseg, s);
    uint32_t rv[kItems];
    double yv[kItems];
    load_rows_y(a, p0, (int64_t)T, y32, true, rv, yv);
    uint32_t gbyte = 0u;
    AggP run = agg_ident();  // trailing run of the lane
    int lastL = -1, lastR = -1;
    {
      uint32_t sc = s;
      SegLite g2 = sg;
#pragma unroll
      for (int j = 0; j < kItems; ++j) {
        const uint64_t p = (uint64_t)p0 + j;
        if (p < T) {
          if (p >= g2.end) {
            sc = seg_gallop(a.pseg, sc + 1u, nseg - 1u, p);
            g2 = seg_lite(a.pseg, sc);
          }
          if (p == g2.start) {
            run = agg_ident();
            run.flag = 1u;
            lastL = lastR = -1;
          }
          if (g2.flags & PS_SPLIT) {
            const uint32_t g = (g2.flags & PS_ALLLEFT) ? 1u : ((bits[rv[j] >> 5] >> (rv[j] & 31)) & 1u);
            gbyte |= g << j;
            if (g) {
              run.nl += 1u;
              run.sl = __dadd_rn(run.sl, __dsub_rn(yv[j], g2.c0));
              lastL = j;
            } else {
              run.sr = __dadd_rn(run.sr, __dsub_rn(yv[j], g2.c1));
              lastR = j;
            }
          }
        }
      }
    }
    if (lastL >= 0) run.xl = a.lx[p0 + lastL];
    if (lastR >= 0) run.xr = a.lx[p0 + lastR];
    AggP wagg;
    const AggP ex = warp_excl_seg(run, agg_ident(), wagg);
    a.gm[cbase / 8 + lane] = (uint8_t)gbyte;
    if (lane == 0) a.agg[ch] = wagg;
    if (kTails) {
      // per split segment ending in this lane: its aggregate from max(segment start,
      // chunk start) to its last entry (the boundary pass adds the chunk carry)
      uint32_t sc = s;
      SegLite g2 = sg;
      AggP r = ex;  // the open segment's part before this lane
      int lL = -1, lR = -1;
#pragma unroll
      for (int j = 0; j < kItems; ++j) {
        const uint64_t p = (uint64_t)p0 + j;
        if (p < T) {
          if (p >= g2.end) {
            sc = seg_gallop(a.pseg, sc + 1u, nseg - 1u, p);
            g2 = seg_lite(a.pseg, sc);
          }
          if (p == g2.start) {
            r = agg_ident();
            r.flag = 1u;
            lL = lR = -1;
          }
          if (g2.flags & PS_SPLIT) {
            if ((gbyte >> j) & 1u) {
              r.nl += 1u;
              r.sl = __dadd_rn(r.sl, __dsub_rn(yv[j], g2.c0));
              lL = j;
            } else {
              r.sr = __dadd_rn(r.sr, __dsub_rn(yv[j], g2.c1));
              lR = j;
            }
            if (p + 1 == g2.end) {
              AggP t = r;
              if (lL >= 0) t.xl = a.lx[p0 + lL];
              if (lR >= 0) t.xr = a.lx[p0 + lR];
              a.tails[sc] = t;
            }
          }
        }
      }
    }
  }
}

// ----------------------------------------------------------------------------- F_B --

// Exclusive segmented scan of the chunk aggregates inside blocks of kBlockChunks chunks,
// then -- by the last block to finish (ticket) -- the exclusive scan of the block
// aggregates (block carries).  Fixed shape: deterministic.
__device__ __forceinline__ AggP block_excl_agg(AggP v, AggP& bagg, AggP* sh) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int nw = blockDim.x >> 5;
  AggP inc = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    AggP o = shfl_up(inc, d);
    if (lane >= d) inc = combine(o, inc);
  }
  if (lane == 31) sh[w] = inc;
  __syncthreads();
  if (w == 0) {
    AggP wv = (lane < nw) ? sh[lane] : agg_ident();
    AggP wi = wv;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      AggP o = shfl_up(wi, d);
      if (lane >= d) wi = combine(o, wi);
    }
    AggP ex = shfl_up(wi, 1);
    if (lane == 0) ex = agg_ident();
    __syncwarp();
    if (lane < nw) sh[lane] = ex;
    if (lane == nw - 1) sh[nw] = wi;
  }
  __syncthreads();
  const AggP wpre = sh[w];
  bagg = sh[nw];
  AggP ex = shfl_up(inc, 1);
  AggP res = (lane == 0) ? wpre : combine(wpre, ex);
  __syncthreads();
  return res;
}

__device__ __forceinline__ AggP ld_cg_agg(const AggP* p) {
  AggP r;
  r.flag = __ldcg(&p->flag);
  r.nl = __ldcg(&p->nl);
  r.sl = __ldcg(&p->sl);
  r.sr = __ldcg(&p->sr);
  r.xl = __ldcg(&p->xl);
  r.xr = __ldcg(&p->xr);
  return r;
}

__device__ __forceinline__ float resolve_x(float v, const float* __restrict__ lx, int64_t c) {
  const uint32_t u = __float_as_uint(v);
  return (u & 0xFFFFFF00u) == kXMark ? __ldg(lx + c * kChunkW + (u & 0xFFu)) : v;
}

__global__ void __launch_bounds__(1024) agg_scan_kernel(Ctl* ctl, int par, const AggP* __restrict__ agg,
                                                       AggP* __restrict__ cexcl, AggP* bagg, AggP* __restrict__ bcarry,
                                                       const float* __restrict__ lx) {
  __shared__ AggP sh[33];
  __shared__ AggP sh_run;
  __shared__ bool s_last;
  const bool full = ctl->nsrch > 0;
  const uint64_t T = full ? ctl->T[par] : 0;  // carries are only used when children are searched
  const int64_t nch = (int64_t)((T + kChunkW - 1) / kChunkW);
  const int64_t b0 = (int64_t)blockIdx.x * kBlockChunks;
  if (b0 < nch) {  // block-uniform
    const int64_t c = b0 + threadIdx.x;
    AggP v = (c < nch) ? agg[c] : agg_ident();
    if (c < nch) {
      v.xl = resolve_x(v.xl, lx, c);
      v.xr = resolve_x(v.xr, lx, c);
    }
    AggP ba;
    const AggP ex = block_excl_agg(v, ba, sh);
    if (c < nch) cexcl[c] = ex;
    if (threadIdx.x == 0) bagg[blockIdx.x] = ba;
  }
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) s_last = atomicAdd(&ctl->ticket, 1u) == gridDim.x - 1;
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  if (threadIdx.x == 0) {
    ctl->ticket = 0u;
    sh_run = agg_ident();
  }
  const int64_t nb = (nch + kBlockChunks - 1) / kBlockChunks;
  __syncthreads();
  for (int64_t base = 0; base < nb; base += blockDim.x) {
    const int64_t bi = base + threadIdx.x;
    const AggP v = (bi < nb) ? ld_cg_agg(bagg + bi) : agg_ident();
    AggP chunk;
    const AggP ex = block_excl_agg(v, chunk, sh);
    const AggP run = sh_run;
    if (bi < nb) bcarry[bi] = combine(run, ex);
    __syncthreads();
    if (threadIdx.x == 0) sh_run = combine(run, chunk);
    __syncthreads();
  }
}

// ----------------------------------------------------------------------------- F_C --

struct FusedArgs {
  const float* lx;
  const uint32_t* lr;
  const double* ly;
  float* ox;
  uint32_t* orow;
  double* oy;
  const uint32_t* desc;
  uint32_t* desc_next;
  const PSeg* pseg;
  const uint8_t* gm;
  const AggP* cexcl;
  const AggP* bcarry;
  Cand2* head_cand;
  Cand2* cont_cand;
  unsigned long long* slot_gain;
  Stat* head_stat;
  Stat* cont_stat;
  const uint2* unit_list;    // {chunk, segment}: a split segment's piece of a chunk
  const uint32_t* small_list;  // split segments of at most kSmallSeg entries (fused_small_kernel)
  Ctl* ctl;
  int par;
  uint32_t level;   // level of the children (written into the pieces)
  uint32_t d;       // lists per level (segments of the parent level: K * d)
  uint32_t m;       // min_samples_leaf (clamped)
  uint32_t ystride; // bytes of one y entry (4 or 8)
  uint32_t stage_bytes;
};

// Stage layout (bytes): x[256] f32 | row[256] u32 | y[256] (4 or 8 B) | gm[32] | PSeg |
// chunk carry | block carry | meta.
constexpr uint32_t kOffX = 0, kOffR = 1024, kOffY = 2048;
__device__ __forceinline__ uint32_t off_gm(uint32_t yb) { return kOffY + 256u * yb; }
__device__ __forceinline__ uint32_t off_ps(uint32_t yb) { return off_gm(yb) + 32u; }
__device__ __forceinline__ uint32_t off_ce(uint32_t yb) { return off_ps(yb) + (uint32_t)sizeof(PSeg); }
__device__ __forceinline__ uint32_t off_cb(uint32_t yb) { return off_ce(yb) + 32u; }
__device__ __forceinline__ uint32_t off_meta(uint32_t yb) { return off_cb(yb) + 32u; }
__host__ __device__ constexpr uint32_t stage_bytes_for(uint32_t yb) { return 2048u + 256u * yb + 32u + (uint32_t)sizeof(PSeg) + 64u + 16u; }

struct Meta {
  int64_t ch;
  uint32_t skip, pad;
};

struct StatQ {
  uint32_t flag;
  double sse, ymin, ymax, s1;
};
__device__ __forceinline__ StatQ statq_ident() { return StatQ{0u, 0.0, INFINITY, -INFINITY, 0.0}; }
__device__ __forceinline__ void stat_add(StatQ& st, double y, double v, double c) {
  const double e = __dsub_rn(y, v);
  st.sse = __dadd_rn(st.sse, __dmul_rn(e, e));
  st.ymin = fmin(st.ymin, y);
  st.ymax = fmax(st.ymax, y);
  st.s1 = __dadd_rn(st.s1, __dsub_rn(y, c));
}

__device__ __forceinline__ void put_cand(const FusedArgs& a, bool head, int64_t ch, int side, uint32_t cs,
                                         double gain, double sl, double thr, uint32_t j) {
  Cand2 c;
  c.gain = gain;
  c.sl = sl;
  c.thr = thr;
  c.j = j;
  c.sp = cs;
  c.level = a.level;
  c.pad = 0u;
  if (head) a.head_cand[cs] = c;
  else a.cont_cand[2 * ch + side] = c;
  atomicMax(a.slot_gain + cs, (unsigned long long)__double_as_longlong(gain));
}
__device__ __forceinline__ void put_stat(const FusedArgs& a, bool head, int64_t ch, int side, uint32_t kc,
                                         const StatQ& q) {
  Stat s{q.sse, q.ymin, q.ymax, q.s1};
  if (head) a.head_stat[kc] = s;
  else a.cont_stat[2 * ch + side] = s;
}


// Loads the plan fields of segment s (global memory; general path).
struct SegCtx {
  uint64_t start, end;
  uint32_t flags, kid;
  int32_t f;
  uint32_t cs[2];
  uint64_t os[2];
  double c[2], v[2], sc[2], soff[2];
  uint32_t N[2], ioff[2];
  float xp[2];
};
__device__ __forceinline__ void load_ctx(SegCtx& c, const PSeg* __restrict__ P) {
  c.start = __ldg(&P->start);
  c.end = c.start + __ldg(&P->cnt);
  c.flags = __ldg(&P->flags);
  c.kid = __ldg(&P->kid);
  c.f = __ldg(&P->f);
#pragma unroll
  for (int q = 0; q < 2; ++q) {
    c.cs[q] = __ldg(&P->cs[q]);
    c.os[q] = __ldg(&P->ostart[q]);
    c.c[q] = __ldg(&P->c[q]);
    c.v[q] = __ldg(&P->v[q]);
    c.sc[q] = __ldg(&P->sc[q]);
    c.soff[q] = __ldg(&P->soff[q]);
    c.N[q] = __ldg(&P->N[q]);
    c.ioff[q] = __ldg(&P->ioff[q]);
    c.xp[q] = __ldg(&P->xprev[q]);
  }
}

__device__ __forceinline__ void store_entry(const FusedArgs& a, bool y32, uint64_t dst, float x, uint32_t r,
                                            const unsigned char* ysrc, uint32_t cs) {
  a.ox[dst] = x;
  a.orow[dst] = r;
  if (y32) reinterpret_cast<uint32_t*>(a.oy)[dst] = *reinterpret_cast<const uint32_t*>(ysrc);
  else reinterpret_cast<unsigned long long*>(a.oy)[dst] = *reinterpret_cast<const unsigned long long*>(ysrc);
  if ((dst & (kChunkW - 1)) == 0) a.desc_next[dst / kChunkW] = cs;
}

// Row-wise stores of one fast chunk (lane = column of a row of 32 entries): left entries
// to the left child's run, right entries to the right child's, both in order.  Returns
// the left count through the chunk (segment-local).
template <bool kY32>
__device__ __forceinline__ uint32_t store_rows(const FusedArgs& a, const PSeg& ps, const uint32_t* w, uint32_t pre,
                                               uint32_t ib, int e_lo, int e_hi, const float* sx, const uint32_t* sr,
                                               const unsigned char* sy, bool w0, bool w1) {
  using YT = typename std::conditional<kY32, uint32_t, unsigned long long>::type;
  const int lane = threadIdx.x & 31;
  const uint32_t lt = (1u << lane) - 1u;
  float* const x0 = a.ox + ps.ostart[0];
  float* const x1 = a.ox + ps.ostart[1];
  uint32_t* const r0 = a.orow + ps.ostart[0];
  uint32_t* const r1 = a.orow + ps.ostart[1];
  YT* const y0 = reinterpret_cast<YT*>(a.oy) + ps.ostart[0];
  YT* const y1 = reinterpret_cast<YT*>(a.oy) + ps.ostart[1];
  const YT* const ys = reinterpret_cast<const YT*>(sy);
#pragma unroll
  for (int r = 0; r < kItems; ++r) {
    const int e = 32 * r + lane;
    const bool in = e >= e_lo && e < e_hi;
    const uint32_t wr = w[r] & __ballot_sync(0xffffffffu, in);  // left entries of this segment
    const bool g = (wr >> lane) & 1u;
    const uint32_t rk = pre + __popc(wr & lt);
    // segment-local index of entry e: ib + e (mod 2^32); right position = index - lefts before
    const uint32_t off = g ? rk : ib + (uint32_t)e - rk;
    if (in && (g ? w0 : w1)) {
      (g ? x0 : x1)[off] = sx[e];
      (g ? r0 : r1)[off] = sr[e];
      (g ? y0 : y1)[off] = ys[e];
    }
    pre += __popc(wr);
  }
  return pre;
}


// y storage (int32 or f64, Reading R24) is decided on the device (root statistics): the
// stage always has room for f64 entries; int32 lists copy and read half of it.
// Work: the fast chunks listed by chunk_plan_kernel (whole chunk inside one segment of a
// split node); a warp per chunk, kStages bulk-copy stages in flight per warp.
__global__ void __launch_bounds__(kFusedThreads, DT_FUSED_MINB) fused_kernel(FusedArgs a) {
  extern __shared__ __align__(128) unsigned char fsm[];
  constexpr uint32_t YB = 8u;
  constexpr uint32_t SB = (stage_bytes_for(YB) + 127u) & ~127u;
  constexpr int kWarps = kFusedThreads / 32;
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  unsigned char* my = fsm + (size_t)wib * kStages * SB;
  uint64_t* bar = reinterpret_cast<uint64_t*>(fsm + (size_t)kWarps * kStages * SB) + wib * kStages;
  PSeg* cur = reinterpret_cast<PSeg*>(fsm + (size_t)kWarps * kStages * SB + kWarps * kStages * sizeof(uint64_t)) + wib;
  const bool full = a.ctl->nsrch > 0;
  const int64_t nfast = a.ctl->nunit;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  if (blockIdx.x == 0 && threadIdx.x == 0) {  // for piece_pos: the chunks of this pass
    const uint64_t Tw = full ? a.ctl->T[a.par] : a.ctl->T0[a.par];
    a.ctl->nch_last = (uint32_t)((Tw + kChunkW - 1) / kChunkW);
  }
  if (gw >= nfast) return;  // warp-uniform; no block barriers below
  const uint32_t m = a.m;
  const uint32_t ilo = m > 1u ? m : 1u;
  const bool y32 = a.ctl->y32 != 0;
  const uint32_t yb = y32 ? 4u : 8u;
  const uint32_t lt = (1u << lane) - 1u;

  auto issue = [&](int s, const uint2 en) {  // lane 0
    unsigned char* st = my + (size_t)s * SB;
    const int64_t ch = (int64_t)en.x;
    reinterpret_cast<Meta*>(st + off_meta(YB))->ch = ch;
    const uint64_t cbase = (uint64_t)ch * kChunkW;
    const uint32_t bytes = 2048u + 256u * yb + 32u + (uint32_t)sizeof(PSeg) + 64u;
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(bar + s, bytes);
    bulk_g2s(st + kOffX, a.lx + cbase, 1024u, bar + s);
    bulk_g2s(st + kOffR, a.lr + cbase, 1024u, bar + s);
    bulk_g2s(st + kOffY, reinterpret_cast<const unsigned char*>(a.ly) + cbase * yb, 256u * yb, bar + s);
    bulk_g2s(st + off_gm(YB), a.gm + cbase / 8, 32u, bar + s);
    bulk_g2s(st + off_ps(YB), a.pseg + en.y, (uint32_t)sizeof(PSeg), bar + s);
    bulk_g2s(st + off_ce(YB), a.cexcl + ch, 32u, bar + s);
    bulk_g2s(st + off_cb(YB), a.bcarry + ch / kBlockChunks, 32u, bar + s);
  };
  uint2 ahead = make_uint2(0u, 0u);  // lane 0: the list entry kStages chunks ahead
  if (lane == 0) {
    for (int q = 0; q < kStages; ++q) mbar_init(bar + q, 1);
    mbar_init_fence();
    for (int q = 0; q < kStages; ++q)
      if (gw + q * nw < nfast) issue(q, a.unit_list[gw + q * nw]);
    if (gw + kStages * nw < nfast) ahead = a.unit_list[gw + kStages * nw];
  }
  __syncwarp();
  int s = 0;
  uint32_t phase = 0;
  for (int64_t idx = gw; idx < nfast; idx += nw) {
    mbar_wait(bar + s, phase);
    unsigned char* st = my + (size_t)s * SB;
    const int64_t nxt = idx + kStages * nw;
    const int64_t ch = reinterpret_cast<const Meta*>(st + off_meta(YB))->ch;
    const uint64_t cbase = (uint64_t)ch * kChunkW;
    // the plan of the chunk's segment: kept in this warp's slot (the stage is refilled
    // before the candidates are evaluated)
    if (lane < (int)(sizeof(PSeg) / 16))
      reinterpret_cast<uint4*>(cur)[lane] = reinterpret_cast<const uint4*>(st + off_ps(YB))[lane];
    __syncwarp();
    const PSeg& ps = *cur;
    const float* sx = reinterpret_cast<const float*>(st + kOffX);
    const uint32_t* sr = reinterpret_cast<const uint32_t*>(st + kOffR);
    const unsigned char* sy = st + kOffY;
    const uint8_t* sgm = st + off_gm(YB);
    const uint4 wq0 = reinterpret_cast<const uint4*>(sgm)[0], wq1 = reinterpret_cast<const uint4*>(sgm)[1];
    const uint32_t w[kItems] = {wq0.x, wq0.y, wq0.z, wq0.w, wq1.x, wq1.y, wq1.z, wq1.w};
    // this segment's entries of the chunk: [e_lo, e_hi) (the whole chunk unless segment
    // heads lie inside; chunk_plan_kernel lists such a chunk once per segment piece)
    const bool headc = ps.start >= cbase;  // the segment's head lies in this chunk
    const int e_lo = headc ? (int)(ps.start - cbase) : 0;
    const int e_hi = (int)min((uint64_t)kChunkW, ps.start + ps.cnt - cbase);
    AggP carry = agg_ident();
    if (full && !headc) carry = combine(*reinterpret_cast<const AggP*>(st + off_cb(YB)),
                                        *reinterpret_cast<const AggP*>(st + off_ce(YB)));
    // lane items
    float xv[kItems];
    double yv[kItems];
    {
      const float4* x4 = reinterpret_cast<const float4*>(sx + lane * kItems);
      const float4 q0 = x4[0], q1 = x4[1];
      xv[0] = q0.x; xv[1] = q0.y; xv[2] = q0.z; xv[3] = q0.w;
      xv[4] = q1.x; xv[5] = q1.y; xv[6] = q1.z; xv[7] = q1.w;
      if (y32) {
        const int4* y4 = reinterpret_cast<const int4*>(sy) + lane * 2;
        const int4 r0 = y4[0], r1 = y4[1];
        yv[0] = r0.x; yv[1] = r0.y; yv[2] = r0.z; yv[3] = r0.w;
        yv[4] = r1.x; yv[5] = r1.y; yv[6] = r1.z; yv[7] = r1.w;
      } else {
        const double2* y2 = reinterpret_cast<const double2*>(sy) + lane * 4;
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const double2 t = y2[q];
          yv[2 * q] = t.x;
          yv[2 * q + 1] = t.y;
        }
      }
    }
    // in-range mask of my items; left / right items of this segment
    uint32_t mbyte;
    {
      const int lo_i = min(max(e_lo - lane * kItems, 0), kItems);
      const int hi_i = min(max(e_hi - lane * kItems, 0), kItems);
      mbyte = ((1u << hi_i) - 1u) & ~((1u << lo_i) - 1u);
    }
    const uint32_t graw = sgm[lane];  // go-left bits of my 8 items (byte lane of w)
    const uint32_t lbyte = graw & mbyte, rbyte = ~graw & mbyte;
    const uint32_t flags = ps.flags;
    const uint32_t ib = (uint32_t)(cbase - ps.start);  // segment-local index of entry 0 (mod 2^32)
    // ---- partition: row-wise coalesced stores (row r = entries 32r .. 32r+31); each
    // child's entries of a row are consecutive
    if (full && (flags & (PS_WR0 | PS_WR1))) {
      const bool w0 = (flags & PS_WR0) != 0, w1 = (flags & PS_WR1) != 0;
      const uint32_t pre = y32 ? store_rows<true>(a, ps, w, carry.nl, ib, e_lo, e_hi, sx, sr, sy, w0, w1)
                               : store_rows<false>(a, ps, w, carry.nl, ib, e_lo, e_hi, sx, sr, sy, w0, w1);
      // chunk descriptors of the next level: a child's run of this piece (<= 256 entries)
      // crossing a multiple of kChunkW starts that chunk of the child's list
      if (lane < 2) {
        const bool g = lane == 0;
        const uint32_t nL = pre - carry.nl, nR = (uint32_t)(e_hi - e_lo) - nL;
        const uint64_t lo = g ? ps.ostart[0] + carry.nl : ps.ostart[1] + (uint64_t)(ib + (uint32_t)e_lo - carry.nl);
        const uint64_t hi = lo + (g ? nL : nR);
        const uint64_t b0 = (lo + kChunkW - 1) & ~(uint64_t)(kChunkW - 1);
        if ((g ? w0 : w1) && b0 < hi) a.desc_next[b0 / kChunkW] = ps.cs[g ? 0 : 1];
      }
    }
    // ---- a chunk (piece) of one x value (few-valued columns: GPU descriptors): no prefix
    // sums are needed -- a child's only possible split position in it is its first item
    // (x there differs from the child's previous x iff the carried x is smaller), whose
    // S'_L is the chunk carry, and the statistics come from feature 0 only (ps.f != 0)
    if (full && ps.f != 0 && sx[e_lo] == sx[e_hi - 1]) {
      const bool anyL = __ballot_sync(0xffffffffu, lbyte != 0u) != 0u;
      const bool anyR = __ballot_sync(0xffffffffu, rbyte != 0u) != 0u;
      const float xc = sx[e_lo];
      __syncwarp();  // the stage is read completely: refill it
      if (lane == 0) {
        if (nxt < nfast) issue(s, ahead);
        if (nxt + nw < nfast) ahead = a.unit_list[nxt + nw];
      }
      const int sd = lane;
      if (lane < 2 && (flags & (sd ? PS_SRCH1 : PS_SRCH0)) && (sd ? anyR : anyL)) {
        float xp = sd ? carry.xr : carry.xl;
        if (isnan(xp)) xp = ps.xprev[sd];
        // the child's items before this one: lefts before the chunk, or rights before it
        const uint32_t jl = sd ? ib + (uint32_t)e_lo - carry.nl : carry.nl;
        const uint32_t io = ps.ioff[sd];
        const uint32_t lo = ilo > io ? ilo - io : 0u;
        const uint32_t hi = ps.N[sd] >= m + io ? ps.N[sd] - m - io + 1u : 0u;
        if (jl >= lo && jl < hi && xp < xc) {
          // S'_L exactly as the item scan forms it: carry + (+0.0 lane prefix)
          const double S = __dadd_rn(ps.soff[sd], __dadd_rn(sd ? carry.sr : carry.sl, 0.0));
          const double gn = split_gain_d(S, ps.sc[sd], (double)(io + jl), (double)ps.N[sd]);
          put_cand(a, headc, ch, sd, ps.cs[sd], gn, S, mid_threshold(xp, xc), io + jl);
        }
      }
      if (++s == kStages) { s = 0; phase ^= 1u; }
      continue;
    }
    // ---- left count before my items, neighbour x across lanes
    uint32_t nl = carry.nl;
    {
      uint32_t cnt = __popc(lbyte);
#pragma unroll
      for (int dd = 1; dd < 32; dd <<= 1) {
        const uint32_t o = __shfl_up_sync(0xffffffffu, cnt, dd);
        if (lane >= dd) cnt += o;
      }
      nl += cnt - __popc(lbyte);
    }
    const uint32_t Lm = __ballot_sync(0xffffffffu, lbyte != 0u) & lt;
    const uint32_t Rm = __ballot_sync(0xffffffffu, rbyte != 0u) & lt;
    float xl = carry.xl, xr = carry.xr;
    {
      // x of the last left / right item of the nearest lower lane holding one
      const int hl = Lm ? 31 - __clz(Lm) : 0, hr = Rm ? 31 - __clz(Rm) : 0;
      const uint32_t bl = __shfl_sync(0xffffffffu, lbyte, hl), br = __shfl_sync(0xffffffffu, rbyte, hr);
      if (Lm) xl = sx[8 * hl + 31 - __clz(bl)];
      if (Rm) xr = sx[8 * hr + 31 - __clz(br)];
    }
    if (isnan(xl)) xl = ps.xprev[0];
    if (isnan(xr)) xr = ps.xprev[1];
    __syncwarp();  // the stage is read completely: refill it
    if (lane == 0) {
      if (nxt < nfast) issue(s, ahead);
      if (nxt + nw < nfast) ahead = a.unit_list[nxt + nw];
    }
    // ---- children's prefix sums: lane sums, Kogge-Stone across lanes, chunk carry
    const double c0 = ps.c[0], c1 = ps.c[1];
    double dv[kItems];
    double sl = 0.0, srr = 0.0;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
      const bool g = (lbyte >> j) & 1u, r = (rbyte >> j) & 1u;
      dv[j] = __dsub_rn(yv[j], g ? c0 : c1);
      // adding +0.0 is exact: a sum of (y - c) terms is never -0.0
      sl = __dadd_rn(sl, g ? dv[j] : 0.0);
      srr = __dadd_rn(srr, r ? dv[j] : 0.0);
    }
    // ---- children's statistics from feature 0
    if (ps.f == 0) {
      StatQ q0 = statq_ident(), q1 = statq_ident();
#pragma unroll
      for (int j = 0; j < kItems; ++j) {
        if ((lbyte >> j) & 1u) stat_add(q0, yv[j], ps.v[0], c0);
        if ((rbyte >> j) & 1u) stat_add(q1, yv[j], ps.v[1], c1);
      }
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        q0.sse = __dadd_rn(q0.sse, __shfl_xor_sync(0xffffffffu, q0.sse, off));
        q0.ymin = fmin(q0.ymin, __shfl_xor_sync(0xffffffffu, q0.ymin, off));
        q0.ymax = fmax(q0.ymax, __shfl_xor_sync(0xffffffffu, q0.ymax, off));
        q0.s1 = __dadd_rn(q0.s1, __shfl_xor_sync(0xffffffffu, q0.s1, off));
        q1.sse = __dadd_rn(q1.sse, __shfl_xor_sync(0xffffffffu, q1.sse, off));
        q1.ymin = fmin(q1.ymin, __shfl_xor_sync(0xffffffffu, q1.ymin, off));
        q1.ymax = fmax(q1.ymax, __shfl_xor_sync(0xffffffffu, q1.ymax, off));
        q1.s1 = __dadd_rn(q1.s1, __shfl_xor_sync(0xffffffffu, q1.s1, off));
      }
      if (lane == 0) {
        put_stat(a, headc, ch, 0, ps.kid, q0);
        if (!(flags & PS_ALLLEFT)) put_stat(a, headc, ch, 1, ps.kid + 1, q1);
      }
    }
    double il = sl, ir = srr;
    warp_incl2(il, ir);
    double SL = __shfl_up_sync(0xffffffffu, il, 1), SR = __shfl_up_sync(0xffffffffu, ir, 1);
    if (lane == 0) { SL = 0.0; SR = 0.0; }
    SL = __dadd_rn(carry.sl, SL);
    SR = __dadd_rn(carry.sr, SR);
    // ---- candidates of both children at every valid position of my items
    if (full && (flags & (PS_SRCH0 | PS_SRCH1))) {
      // right position of my first in-range item: its segment-local index - lefts before
      const uint32_t jr0 = ib + (uint32_t)max(lane * kItems, e_lo) - nl;
      // both children in one pass over my items (each item belongs to one child; the
      // child's running state is selected per item: no divergence between the lanes)
      const uint32_t io0 = ps.ioff[0], io1 = ps.ioff[1];
      const uint32_t lo0 = ilo > io0 ? ilo - io0 : 0u, lo1 = ilo > io1 ? ilo - io1 : 0u;
      const uint32_t hi0 = ((flags & PS_SRCH0) && ps.N[0] >= m + io0) ? ps.N[0] - m - io0 + 1u : 0u;
      const uint32_t hi1 = ((flags & PS_SRCH1) && ps.N[1] >= m + io1) ? ps.N[1] - m - io1 + 1u : 0u;
      double S0 = __dadd_rn(ps.soff[0], SL), S1 = __dadd_rn(ps.soff[1], SR);
      uint32_t j0 = nl, j1 = jr0;
      float xp0 = xl, xp1 = xr;
      double bg0 = -1.0, bg1 = -1.0, bs0 = 0.0, bs1 = 0.0;
      uint32_t bj0 = 0xffffffffu, bj1 = 0xffffffffu;
      float bxp0 = 0.f, bx0 = 0.f, bxp1 = 0.f, bx1 = 0.f;
      // exact gain (Reading R19) at every valid position; strict >: lowest position
#pragma unroll
      for (int j = 0; j < kItems; ++j) {
        const bool g = (lbyte >> j) & 1u, r = (rbyte >> j) & 1u;
        const uint32_t jl = g ? j0 : j1;
        const float xp = g ? xp0 : xp1;
        if ((g || r) && jl >= (g ? lo0 : lo1) && jl < (g ? hi0 : hi1) && xp < xv[j]) {
          const double S = g ? S0 : S1;
          const double gn = split_gain_d(S, g ? ps.sc[0] : ps.sc[1], (double)((g ? io0 : io1) + jl),
                                         (double)(g ? ps.N[0] : ps.N[1]));
          if (g) {
            if (gn > bg0) { bg0 = gn; bs0 = S; bj0 = io0 + jl; bxp0 = xp; bx0 = xv[j]; }
          } else {
            if (gn > bg1) { bg1 = gn; bs1 = S; bj1 = io1 + jl; bxp1 = xp; bx1 = xv[j]; }
          }
        }
        if (g) { S0 = __dadd_rn(S0, dv[j]); ++j0; xp0 = xv[j]; }
        if (r) { S1 = __dadd_rn(S1, dv[j]); ++j1; xp1 = xv[j]; }
      }
#pragma unroll 1
      for (int side = 0; side < 2; ++side) {
        if (!(flags & (side ? PS_SRCH1 : PS_SRCH0))) continue;  // warp-uniform
        const double bg = side ? bg1 : bg0;
        const uint32_t bj = side ? bj1 : bj0;
        // warp max of the exact gains (>= 0: the f64 bit patterns order like the values;
        // key 0 = no candidate), then the lowest position holding it
        const unsigned long long key = bg >= 0.0 ? (unsigned long long)__double_as_longlong(bg) + 1ull : 0ull;
        const uint32_t khi = __reduce_max_sync(0xffffffffu, (uint32_t)(key >> 32));
        const uint32_t klo = __reduce_max_sync(0xffffffffu, (uint32_t)(key >> 32) == khi ? (uint32_t)key : 0u);
        const unsigned long long kmax = ((unsigned long long)khi << 32) | klo;
        if (kmax != 0ull) {
          const uint32_t jmin = __reduce_min_sync(0xffffffffu, key == kmax ? bj : 0xffffffffu);
          if (key == kmax && bj == jmin)  // exactly one lane holds the winner
            put_cand(a, headc, ch, side, ps.cs[side], bg, side ? bs1 : bs0,
                     side ? mid_threshold(bxp1, bx1) : mid_threshold(bxp0, bx0), jmin);
        }
      }
    }
    if (++s == kStages) { s = 0; phase ^= 1u; }
  }
}

// F_C for the split segments of at most kSmallSeg entries (small list of chunk_plan_kernel):
// a warp per segment, lane i = entry start + i.  The segment is one (head) piece: its
// children's ranks are ballots, their prefix sums Kogge-Stone scans of the lanes, every
// valid position is evaluated with the exact gain (Reading R19) and the lowest position of
// the highest gain per child is recorded.  When the segment straddles a chunk boundary
// the continuation statistics slot of its second chunk gets the identity.
__global__ void __launch_bounds__(kThreads) fused_small_kernel(FusedArgs a) {
  const int lane = threadIdx.x & 31;
  const int64_t ns = a.ctl->nsmall;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const bool full = a.ctl->nsrch > 0;
  const bool y32 = a.ctl->y32 != 0;
  const uint32_t m = a.m;
  const uint32_t ilo = m > 1u ? m : 1u;
  const uint32_t lt = (1u << lane) - 1u;
  for (int64_t idx = gw; idx < ns; idx += nw) {
    SegCtx cx;
    load_ctx(cx, a.pseg + a.small_list[idx]);
    const uint32_t cnt = (uint32_t)(cx.end - cx.start);
    const bool in = (uint32_t)lane < cnt;
    const uint64_t p = cx.start + (uint64_t)lane;
    float x = 0.f;
    uint32_t row = 0u;
    unsigned long long yraw = 0ull;
    double y = 0.0;
    bool g = false;
    if (in) {
      x = a.lx[p];
      row = a.lr[p];
      if (y32) {
        const int32_t yi = reinterpret_cast<const int32_t*>(a.ly)[p];
        yraw = (uint32_t)yi;
        y = (double)yi;
      } else {
        yraw = reinterpret_cast<const unsigned long long*>(a.ly)[p];
        y = __longlong_as_double((long long)yraw);
      }
      g = ((a.gm[p >> 3] >> (p & 7u)) & 1u) != 0u;
    }
    const int side = g ? 0 : 1;
    const uint32_t Lb = __ballot_sync(0xffffffffu, in && g), Rb = __ballot_sync(0xffffffffu, in && !g);
    const uint32_t mine = g ? Lb : Rb;
    const uint32_t jl = __popc(mine & lt);  // my child's entries before mine (this rank)
    // ---- partition: my child's run, in order
    if (full && in && (cx.flags & (side ? PS_WR1 : PS_WR0))) {
      const uint64_t dst = (side ? cx.os[1] : cx.os[0]) + jl;
      a.ox[dst] = x;
      a.orow[dst] = row;
      if (y32) reinterpret_cast<uint32_t*>(a.oy)[dst] = (uint32_t)yraw;
      else reinterpret_cast<unsigned long long*>(a.oy)[dst] = yraw;
      if ((dst & (kChunkW - 1)) == 0) a.desc_next[dst / kChunkW] = (side ? cx.cs[1] : cx.cs[0]);
    }
    // ---- children's statistics from feature 0
    if (cx.f == 0) {
      StatQ q0 = statq_ident(), q1 = statq_ident();
      if (in) {
        if (g) stat_add(q0, y, cx.v[0], cx.c[0]);
        else stat_add(q1, y, cx.v[1], cx.c[1]);
      }
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        q0.sse = __dadd_rn(q0.sse, __shfl_xor_sync(0xffffffffu, q0.sse, off));
        q0.ymin = fmin(q0.ymin, __shfl_xor_sync(0xffffffffu, q0.ymin, off));
        q0.ymax = fmax(q0.ymax, __shfl_xor_sync(0xffffffffu, q0.ymax, off));
        q0.s1 = __dadd_rn(q0.s1, __shfl_xor_sync(0xffffffffu, q0.s1, off));
        q1.sse = __dadd_rn(q1.sse, __shfl_xor_sync(0xffffffffu, q1.sse, off));
        q1.ymin = fmin(q1.ymin, __shfl_xor_sync(0xffffffffu, q1.ymin, off));
        q1.ymax = fmax(q1.ymax, __shfl_xor_sync(0xffffffffu, q1.ymax, off));
        q1.s1 = __dadd_rn(q1.s1, __shfl_xor_sync(0xffffffffu, q1.s1, off));
      }
      if (lane == 0) {
        put_stat(a, true, 0, 0, cx.kid, q0);
        if (!(cx.flags & PS_ALLLEFT)) put_stat(a, true, 0, 1, cx.kid + 1, q1);
        const int64_t c0 = (int64_t)(cx.start / kChunkW), c1 = (int64_t)((cx.end - 1) / kChunkW);
        if (c1 > c0) {
          const Stat z{0.0, INFINITY, -INFINITY, 0.0};
          a.cont_stat[2 * c1] = z;
          a.cont_stat[2 * c1 + 1] = z;
        }
      }
    }
    if (!full || !(cx.flags & (PS_SRCH0 | PS_SRCH1))) continue;  // warp-uniform
    // ---- prefix sums of (y - c_child) over my child's earlier entries (exclusive: the
    // inclusive scan of the lane below; non-members add +0.0, exact)
    const double dv = in ? __dsub_rn(y, side ? cx.c[1] : cx.c[0]) : 0.0;
    double il = (in && g) ? dv : 0.0, ir = (in && !g) ? dv : 0.0;
    warp_incl2(il, ir);
    double el = __shfl_up_sync(0xffffffffu, il, 1), er = __shfl_up_sync(0xffffffffu, ir, 1);
    if (lane == 0) el = er = 0.0;
    // x of my child's previous entry (this rank), else the rank carry (NaN: none)
    const uint32_t below = mine & lt;
    const float xo = __shfl_sync(0xffffffffu, x, below ? 31 - __clz(below) : 0);
    const float xp = below ? xo : (side ? cx.xp[1] : cx.xp[0]);
    // ---- my position's candidate (as fused_kernel: valid local range [lo, hi), x_prev < x)
    double gain = -1.0, S = 0.0;
    const uint32_t io = (side ? cx.ioff[1] : cx.ioff[0]), Nc = (side ? cx.N[1] : cx.N[0]);
    if (in && (cx.flags & (side ? PS_SRCH1 : PS_SRCH0))) {
      const uint32_t lo = ilo > io ? ilo - io : 0u;
      const uint32_t hi = Nc >= m + io ? Nc - m - io + 1u : 0u;
      S = __dadd_rn((side ? cx.soff[1] : cx.soff[0]), side ? er : el);
      if (jl >= lo && jl < hi && xp < x) gain = split_gain_d(S, (side ? cx.sc[1] : cx.sc[0]), (double)(io + jl), (double)Nc);
    }
    const uint32_t jg = io + jl;
#pragma unroll 1
    for (int sd = 0; sd < 2; ++sd) {
      if (!(cx.flags & (sd ? PS_SRCH1 : PS_SRCH0))) continue;  // warp-uniform
      const unsigned long long key =
          (side == sd && gain >= 0.0) ? (unsigned long long)__double_as_longlong(gain) + 1ull : 0ull;
      const uint32_t khi = __reduce_max_sync(0xffffffffu, (uint32_t)(key >> 32));
      const uint32_t klo = __reduce_max_sync(0xffffffffu, (uint32_t)(key >> 32) == khi ? (uint32_t)key : 0u);
      const unsigned long long kmax = ((unsigned long long)khi << 32) | klo;
      if (kmax == 0ull) continue;
      const uint32_t jmin = __reduce_min_sync(0xffffffffu, key == kmax ? jg : 0xffffffffu);
      if (key == kmax && jg == jmin)
        put_cand(a, true, 0, sd, (sd ? cx.cs[1] : cx.cs[0]), gain, S, mid_threshold(xp, x), jg);
    }
  }
}

}  // namespace

// ------------------------------------------------------------------------ launchers --

namespace {
int grid_for(const void* kern, int threads, size_t smem) {
  int per = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, kern, threads, smem);
  if (per < 1) per = 1;
  return num_sms() * per;
}
constexpr int64_t kMaxSmemBits = 227 * 1024;
}  // namespace

// F_A + F_B of the pass whose parent level is la.level (la.level = -1: the virtual root).
dt_status level_agg_enqueue(const FitBufs& b, const LevelArgs& la, cudaStream_t s) {
  AggArgs a;
  a.walk_gen = la.level < 0 || la.tails;
  a.lr = b.lr[la.cur];
  a.ly = b.ly[la.cur];
  a.lx = b.lx[la.cur];
  a.desc = b.desc[la.par];
  a.pseg = b.pseg;
  a.gbits = b.gbits;
  a.gm = b.gm;
  a.agg = b.agg;
  a.tails = b.tails;
  a.fast_list = b.fast_list;
  a.gen_list = b.gen_list;
  a.ctl = b.ctl;
  a.par = la.par;
  a.d = (uint32_t)la.d;
  a.nwords = b.nwords4;
  chunk_plan_kernel<<<num_sms() * 8, 256, 0, s>>>(b.ctl, la.par, la.d, b.desc[la.par], b.pseg, b.agg, b.fast_list,
                                                  b.gen_list, b.unit_list, b.small_list, la.level < 0);
  DT_CK(cudaGetLastError());
  const size_t bytes = sizeof(uint32_t) * (size_t)b.nwords4;
  if ((int64_t)bytes <= kMaxSmemBits) {
    auto k = la.tails ? level_agg_kernel<true, true> : level_agg_kernel<true, false>;
    DT_CK(cudaFuncSetAttribute((const void*)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes));
    k<<<num_sms(), 1024, bytes, s>>>(a);
  } else {
    auto k = la.tails ? level_agg_kernel<false, true> : level_agg_kernel<false, false>;
    k<<<grid_for((const void*)k, kThreads, 0), kThreads, 0, s>>>(a);
  }
  DT_CK(cudaGetLastError());
  agg_scan_kernel<<<(unsigned)b.max_cblocks, kBlockChunks, 0, s>>>(b.ctl, la.par, b.agg, b.cexcl, b.bagg, b.bcarry,
                                                          b.lx[la.cur]);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

size_t fused_smem() {
  const size_t sb = (stage_bytes_for(8u) + 127u) & ~127u;
  constexpr int kWarps = kFusedThreads / 32;
  return sb * kStages * kWarps + kWarps * kStages * sizeof(uint64_t) + kWarps * sizeof(PSeg);
}

// F_C of the pass whose parent level is la.level.
dt_status level_fused_enqueue(const FitBufs& b, const LevelArgs& la, cudaStream_t s) {
  FusedArgs a;
  a.lx = b.lx[la.cur];
  a.lr = b.lr[la.cur];
  a.ly = b.ly[la.cur];
  a.ox = b.lx[la.cur ^ 1];
  a.orow = b.lr[la.cur ^ 1];
  a.oy = b.ly[la.cur ^ 1];
  a.desc = b.desc[la.par];
  a.desc_next = b.desc[la.par ^ 1];
  a.pseg = b.pseg;
  a.gm = b.gm;
  a.cexcl = b.cexcl;
  a.bcarry = b.bcarry;
  a.head_cand = b.head_cand;
  a.cont_cand = b.cont_cand;
  a.slot_gain = b.slot_gain;
  a.head_stat = b.head_stat;
  a.cont_stat = b.cont_stat;
  a.ctl = b.ctl;
  a.par = la.par;
  a.level = (uint32_t)(la.level + 1);
  a.d = (uint32_t)la.d;
  a.m = (uint32_t)std::min<int64_t>(la.min_leaf, 0x7fffffff);
  a.ystride = 0;
  a.stage_bytes = 0;
  const size_t sm = fused_smem();
  a.unit_list = b.unit_list;
  a.small_list = b.small_list;
  auto k = fused_kernel;
  DT_CK(cudaFuncSetAttribute((const void*)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
  k<<<grid_for((const void*)k, kFusedThreads, sm), kFusedThreads, sm, s>>>(a);
  DT_CK(cudaGetLastError());
  fused_small_kernel<<<grid_for((const void*)fused_small_kernel, kThreads, 0), kThreads, 0, s>>>(a);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

}  // namespace dtl
