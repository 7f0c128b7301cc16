// Root statistics and the presort of the exact CART fit (DESIGN.md
// "Kernels"): per-feature stable sort of (x, row id) once per fit, written as the level-0
// lists, the level-0 segment table, the chunk descriptors and the root node.
#include <algorithm>
#include <type_traits>
#include <vector>

#include "fit_core.cuh"

namespace dtl {

namespace {

struct RootPart {
  double s, c;  // Neumaier sum
  double mn, mx;
  int integral, finite;
};

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

// Folds of the block parts in index order (one thread; the parts are staged in shared
// memory by the whole block, 256 at a time, so the fold does not wait on each load).
__global__ void __launch_bounds__(256) root_finalize_kernel(const RootPart* parts, int nparts, int64_t n, Ctl* ctl) {
  __shared__ RootPart sp[256];
  double s = 0, c = 0, mn = INFINITY, mx = -INFINITY;
  int integral = 1, finite = 1;
  for (int i0 = 0; i0 < nparts; i0 += 256) {
    __syncthreads();
    if (i0 + (int)threadIdx.x < nparts) sp[threadIdx.x] = parts[i0 + threadIdx.x];
    __syncthreads();
    if (threadIdx.x == 0) {
      for (int i = 0; i < min(256, nparts - i0); ++i) {
        neu_add(s, c, sp[i].s);
        neu_add(s, c, sp[i].c);
        mn = fmin(mn, sp[i].mn);
        mx = fmax(mx, sp[i].mx);
        integral &= sp[i].integral;
        finite &= sp[i].finite;
      }
    }
  }
  if (threadIdx.x != 0) return;
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
// (n: rows of this call; n_all: rows of the whole table, whose mean gives the centre)
__global__ void __launch_bounds__(256) root_center_kernel(const double* __restrict__ y, int64_t n, int64_t n_all,
                                                          int64_t chunk, const Ctl* ctl, double* parts) {
  const int64_t lo = (int64_t)blockIdx.x * chunk, hi = min(n, lo + chunk);
  double c0;
  if (ctl->int_mode) c0 = (double)floor_div_ll((long long)ctl->ysum, (long long)n_all);
  else c0 = __ddiv_rn(ctl->ysum, (double)n_all);
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

__global__ void __launch_bounds__(256) root_init_kernel(const double* parts, int nparts, int64_t n, int d,
                                                        int32_t max_depth, int64_t min_leaf, Ctl* ctl, NodeL* nodes0,
                                                        Decision* dec_root) {
  __shared__ double sp[256];
  double s = 0, cc = 0;
  for (int i0 = 0; i0 < nparts; i0 += 256) {
    __syncthreads();
    if (i0 + (int)threadIdx.x < nparts) sp[threadIdx.x] = parts[i0 + threadIdx.x];
    __syncthreads();
    if (threadIdx.x == 0)
      for (int i = 0; i < min(256, nparts - i0); ++i) neu_add(s, cc, sp[i]);
  }
  if (threadIdx.x != 0) return;
  NodeL nd;
  nd.N = (uint32_t)n;
  nd.id = 0;
  nd.searchable = (max_depth != 0 && n >= 2 * min_leaf) ? 1 : 0;
  nd.parent = 0;
  if (ctl->int_mode) {
    nd.c = (double)floor_div_ll((long long)ctl->ysum, (long long)n);
    nd.v = __ddiv_rn(ctl->ysum, (double)n);
    nd.sc = ctl->ysum - nd.c * (double)n;  // exact in integer mode
  } else {
    nd.v = __ddiv_rn(ctl->ysum, (double)n);
    nd.c = nd.v;
    nd.sc = __dadd_rn(s, cc);
  }
  nd.side = 0;
  nd.wstart = 0;
  nd.pad[0] = nd.pad[1] = nd.pad[2] = nd.pad[3] = 0;
  nodes0[0] = nd;
  ctl->ysc = nd.sc;
  ctl->T[0] = (unsigned long long)n * (unsigned long long)d;
  ctl->T0[0] = (unsigned long long)n;
  ctl->K[0] = 1;
  ctl->next_id = 1;
  ctl->split_evals = 0;
  ctl->max_depth_seen = 0;
  ctl->nsrch = (uint32_t)nd.searchable;  // the virtual-root pass searches the root's candidates
  Decision dr;
  dr.f = 0;
  dr.nl = (uint32_t)n;
  dr.kid = 0;
  dr.flags = DEC_ALL_LEFT;
  dr.sl = 0.0;
  dr.thr = 0.0;
  *dec_root = dr;
}

// Level-0 tables (one segment per feature list, K = 1), the chunk descriptors of the
// level-0 lists, and the plan of the virtual-root pass: every entry goes "left" to the
// root, nothing is written (the level-0 lists are the presort's output), the root's
// candidates and statistics are evaluated.
__global__ void __launch_bounds__(256) root_tables_kernel(const Ctl* __restrict__ ctl, const NodeL* __restrict__ nodes0,
                                                          int64_t n, int d, SegT* __restrict__ seg0,
                                                          PSeg* __restrict__ pseg, uint32_t* __restrict__ desc0) {
  const NodeL rt = nodes0[0];
  const int64_t nch = (n * d + kChunkW - 1) / kChunkW;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nch; i += (int64_t)gridDim.x * blockDim.x)
    desc0[i] = (uint32_t)((i * kChunkW) / n);
  for (int64_t f = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; f < d; f += (int64_t)gridDim.x * blockDim.x) {
    SegT sg;
    sg.start = (uint64_t)f * (uint64_t)n;
    sg.cnt = (uint32_t)n;
    sg.k = 0;
    sg.f = (int32_t)f;
    sg.ioff = 0;
    sg.soff = 0.0;
    sg.xprev = __int_as_float(0x7fc00000);
    sg.pad = 0;
    seg0[f] = sg;
    PSeg p;
    p.start = sg.start;
    p.cnt = sg.cnt;
    p.k = 0;
    p.f = (int32_t)f;
    p.flags = PS_SPLIT | PS_ALLLEFT | (rt.searchable ? PS_SRCH0 : 0u);
    p.cs[0] = p.cs[1] = (uint32_t)f;
    p.ostart[0] = p.ostart[1] = sg.start;
    p.c[0] = p.c[1] = rt.c;
    p.v[0] = p.v[1] = rt.v;
    p.sc[0] = p.sc[1] = rt.sc;
    p.N[0] = p.N[1] = rt.N;
    p.ioff[0] = p.ioff[1] = 0;
    p.soff[0] = p.soff[1] = 0.0;
    p.xprev[0] = p.xprev[1] = __int_as_float(0x7fc00000);
    p.kid = 0;
    p.glim = 0;
    pseg[f] = p;
  }
  (void)ctl;
}


// Batched LSD radix sort of the d per-feature key lists (any n < 2^32): 4 passes
// of 8-bit digits; per pass three launches, each over all d features (grid.y = feature):
//   rs_count:   per-tile digit counts;
//   rs_offset_warp: per (feature, digit) exclusive scan of the counts over the tiles, and
//               the digit totals (a warp per scan);
//   rs_scatter: every key's stable rank inside its tile (warp match_any per step of 32
//               keys + per-warp digit counters; keys in tile order), then its destination
//               = (keys of smaller digits) + (same digit, earlier tiles) + rank.
// Stable within a feature, so equal keys keep the row order: (x, row id) order (R6).
#ifndef DT_RS_WARPS
#define DT_RS_WARPS 12  // warps per scatter tile (256 keys each): 3072-key tiles (8 warps: 2% slower presort)
#endif
constexpr int kTS = 256, kTI = 8;                    // count: threads per block; keys per scatter thread
constexpr int kSTS = 32 * DT_RS_WARPS;               // scatter: threads per block
constexpr int kTile = kSTS * kTI;                    // keys per tile (count and scatter)

// Source of a pass's keys: the key lists, or (first pass, kFromX) X itself: key =
// flip(X[r][f]), value = row0 + r (the table's columns read in place; the d blocks of a
// tile run side by side, so X's rows are read from L2 once per tile).
template <bool kFromX>
__device__ __forceinline__ uint32_t rs_key(const uint32_t* __restrict__ keys, const float* __restrict__ X, int64_t n,
                                           int d, int f, int64_t i) {
  if (kFromX) return flip_f32(__ldg(X + i * d + f));
  return __ldg(keys + (int64_t)f * n + i);
}

// grid: d x tiles blocks, block b = (feature b % d, tile b / d)
template <bool kFromX>
__global__ void __launch_bounds__(kTS) rs_count_kernel(const uint32_t* __restrict__ keys, const float* __restrict__ X,
                                                       int64_t n, int d, int shift, int tiles,
                                                       uint32_t* __restrict__ cnt, Ctl* ctl) {
  __shared__ uint32_t h[256];
  const int f = (int)(blockIdx.x % (unsigned)d), tile = (int)(blockIdx.x / (unsigned)d);
  h[threadIdx.x] = 0u;
  __syncthreads();
  const int64_t base = (int64_t)tile * kTile;
  const int m = (int)min((int64_t)kTile, n - base);
  bool bad = false;
  for (int i = threadIdx.x; i < m; i += kTS) {
    const uint32_t key = rs_key<kFromX>(keys, X, n, d, f, base + i);
    if (kFromX && !isfinite(unflip_f32(key))) bad = true;  // a6: non-finite X (flip keeps NaN / inf patterns)
    atomicAdd(&h[(key >> shift) & 255u], 1u);
  }
  if (kFromX && __syncthreads_or(bad) && threadIdx.x == 0) ctl->nonfinite = 1;
  __syncthreads();
  cnt[((int64_t)f * 256 + threadIdx.x) * tiles + tile] = h[threadIdx.x];
}

// Exclusive prefix of one (feature, digit)'s counts over the tiles, and the digit's total:
// a warp per scan, 32 tiles per step (lane = tile), a warp inclusive scan plus the running
// carry; the next step's counts are loaded before this step's scan (fixed shape; integers).
__global__ void __launch_bounds__(256) rs_offset_warp_kernel(const uint32_t* __restrict__ cnt, int tiles, int nscan,
                                                             uint32_t* __restrict__ off, uint32_t* __restrict__ tot) {
  const int lane = threadIdx.x & 31;
  const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (wid >= nscan) return;
  const int64_t base = wid * tiles;  // scan wid = feature * 256 + digit
  uint32_t run = 0u;
  uint32_t c = lane < tiles ? __ldg(cnt + base + lane) : 0u;
  for (int t0 = 0; t0 < tiles; t0 += 32) {
    const int t = t0 + lane, tn = t + 32;
    const uint32_t cn = tn < tiles ? __ldg(cnt + base + tn) : 0u;  // next step in flight
    uint32_t inc = c;
#pragma unroll
    for (int dd = 1; dd < 32; dd <<= 1) {
      const uint32_t o = __shfl_up_sync(0xffffffffu, inc, dd);
      if (lane >= dd) inc += o;
    }
    if (t < tiles) off[base + t] = run + inc - c;
    run += __shfl_sync(0xffffffffu, inc, 31);
    c = cn;
  }
  if (lane == 0) tot[wid] = run;
}

#ifndef DT_RS_MINB
#define DT_RS_MINB 3  // CTAs/SM of the scatter: 3 x 384 threads (2: 14% slower presort)
#endif
// kToLists (last pass): the sorted pairs go straight into the level-0 lists: x =
// unflip(key), row = value, y = y[row - row0] (int32 when the fit stores y so, R24).
struct RsOut {
  uint32_t* kout;
  uint32_t* vout;
  float* lx;
  uint32_t* lr;
  double* ly;
  const double* y;
  int64_t row0;
  const Ctl* ctl;
};
template <bool kFromX, bool kToLists>
__global__ void __launch_bounds__(kSTS, DT_RS_MINB) rs_scatter_kernel(const uint32_t* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                         const float* __restrict__ X, int d, RsOut o,
                                                         int64_t n, int shift, int tiles, const uint32_t* __restrict__ off,
                                                         const uint32_t* __restrict__ tot) {
  __shared__ uint32_t wc[kSTS / 32][256];  // per-warp digit counters -> per-warp prefixes
  __shared__ uint32_t s_base[256];        // digit base of this tile: smaller digits + earlier tiles
  __shared__ uint32_t s_start[256];       // digit starts inside the tile
  __shared__ uint32_t skey[kTile], sval[kTile];
  __shared__ uint32_t sw[8], sw2[8];       // digit scans: 256 digits = 8 warps
  const int f = (int)(blockIdx.x % (unsigned)d), tile = (int)(blockIdx.x / (unsigned)d);
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t tbase = (int64_t)tile * kTile;
  const int m = (int)min((int64_t)kTile, n - tbase);
  for (int q = lane; q < 256; q += 32) wc[w][q] = 0u;
  // keys of warp w: tile positions w * 256 + j * 32 + lane (coalesced, in tile order)
  uint32_t keys[kTI], vals[kTI], rk[kTI];
#pragma unroll
  for (int j = 0; j < kTI; ++j) {
    const int i = w * 256 + j * 32 + lane;
    keys[j] = (i < m) ? rs_key<kFromX>(kin, X, n, d, f, tbase + i) : 0u;
    vals[j] = (i < m) ? (kFromX ? (uint32_t)(o.row0 + tbase + i) : __ldg(vin + (int64_t)f * n + tbase + i)) : 0u;
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
    const int dgt = threadIdx.x;  // threads 0..255: one digit each
    uint32_t run = 0u, inc = 0u, t = 0u, tinc = 0u;
    if (dgt < 256) {
#pragma unroll
      for (int q = 0; q < kSTS / 32; ++q) {
        const uint32_t c = wc[q][dgt];
        wc[q][dgt] = run;
        run += c;
      }
      inc = run;  // tile count of this digit
#pragma unroll
      for (int dd = 1; dd < 32; dd <<= 1) {
        const uint32_t o = __shfl_up_sync(0xffffffffu, inc, dd);
        if (lane >= dd) inc += o;
      }
      if (lane == 31) sw[w] = inc;
      // exclusive prefix of the digit totals of this feature
      t = __ldg(tot + (int64_t)f * 256 + dgt);
      tinc = t;
#pragma unroll
      for (int dd = 1; dd < 32; dd <<= 1) {
        const uint32_t o = __shfl_up_sync(0xffffffffu, tinc, dd);
        if (lane >= dd) tinc += o;
      }
      if (lane == 31) sw2[w] = tinc;
    }
    __syncthreads();
    if (dgt < 256) {
      uint32_t wp = 0u, wp2 = 0u;
      for (int q = 0; q < w; ++q) { wp += sw[q]; wp2 += sw2[q]; }
      s_start[dgt] = wp + inc - run;
      s_base[dgt] = wp2 + tinc - t + __ldg(off + ((int64_t)f * 256 + dgt) * tiles + tile);
    }
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
  const bool y32 = kToLists && o.ctl->y32 != 0;
  for (int i = threadIdx.x; i < m; i += kSTS) {
    const uint32_t key = skey[i];
    const uint32_t dg = (key >> shift) & 255u;
    const int64_t dst = (int64_t)f * n + s_base[dg] + ((uint32_t)i - s_start[dg]);
    if (kToLists) {
      const uint32_t r = sval[i];
      o.lx[dst] = unflip_f32(key);
      o.lr[dst] = r;
      const double v = __ldg(o.y + (r - o.row0));
      if (y32) reinterpret_cast<int32_t*>(o.ly)[dst] = (int32_t)v;
      else o.ly[dst] = v;
    } else {
      o.kout[dst] = key;
      o.vout[dst] = sval[i];
    }
  }
}

// ------------------------------------------------------------ value-range sharding --
// (SURVEY 8(e)): rank p of P ends up holding, for every feature f,
// the entries at global sorted positions [p n / P, (p + 1) n / P) of f's (x, row id)
// order: a local sort, exact splitters by bisection on the 64-bit key (flip(x) << 32 |
// row id, all distinct) with a sum-allreduce of the ranks' counts per round, an
// all-to-all of 16-byte entries, a local stable sort of the received runs (source-rank
// order = row order for equal x, since rank q holds rows [row_offset_q, ...)).

struct Sent {  // one entry on the wire
  uint32_t key, row;
  double y;
};

// One rank's partial of the root statistics (block parts folded in index order; staged
// in shared memory as in root_finalize_kernel).
__global__ void __launch_bounds__(256) root_fold_kernel(const RootPart* parts, int nparts, RootPart* out) {
  __shared__ RootPart sp[256];
  RootPart a{0, 0, INFINITY, -INFINITY, 1, 1};
  for (int i0 = 0; i0 < nparts; i0 += 256) {
    __syncthreads();
    if (i0 + (int)threadIdx.x < nparts) sp[threadIdx.x] = parts[i0 + threadIdx.x];
    __syncthreads();
    if (threadIdx.x == 0) {
      for (int i = 0; i < min(256, nparts - i0); ++i) {
        neu_add(a.s, a.c, sp[i].s);
        neu_add(a.s, a.c, sp[i].c);
        a.mn = fmin(a.mn, sp[i].mn);
        a.mx = fmax(a.mx, sp[i].mx);
        a.integral &= sp[i].integral;
        a.finite &= sp[i].finite;
      }
    }
  }
  if (threadIdx.x == 0) *out = a;
}
__global__ void __launch_bounds__(256) center_fold_kernel(const double* parts, int nparts, double* out) {
  __shared__ double sp[256];
  double s = 0, cc = 0;
  for (int i0 = 0; i0 < nparts; i0 += 256) {
    __syncthreads();
    if (i0 + (int)threadIdx.x < nparts) sp[threadIdx.x] = parts[i0 + threadIdx.x];
    __syncthreads();
    if (threadIdx.x == 0)
      for (int i = 0; i < min(256, nparts - i0); ++i) neu_add(s, cc, sp[i]);
  }
  if (threadIdx.x == 0) *out = __dadd_rn(s, cc);
}

__device__ __forceinline__ unsigned long long ckey(const uint32_t* keys, const uint32_t* vals, int64_t i) {
  return ((unsigned long long)keys[i] << 32) | vals[i];
}
// number of local composite keys < v in a sorted list of n
__device__ __forceinline__ uint32_t count_less(const uint32_t* keys, const uint32_t* vals, int64_t n,
                                               unsigned long long v) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    if (ckey(keys, vals, mid) < v) lo = mid + 1;
    else hi = mid;
  }
  return (uint32_t)lo;
}

// bisection state per (feature, boundary b = 1 .. P-1): [lo, hi) with count(< lo) <= t_b
__global__ void split_init_kernel(unsigned long long* lohi, int nb) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nb; i += gridDim.x * blockDim.x) {
    lohi[2 * i] = 0ull;
    lohi[2 * i + 1] = ~0ull;
  }
}
__global__ void split_count_kernel(const uint32_t* __restrict__ keys, const uint32_t* __restrict__ vals, int64_t n,
                                   int nbper, int nb, const unsigned long long* __restrict__ lohi,
                                   unsigned long long* __restrict__ cnt) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nb; i += gridDim.x * blockDim.x) {
    const int f = i / nbper;
    const unsigned long long lo = lohi[2 * i], hi = lohi[2 * i + 1];
    const unsigned long long mid = lo + (hi - lo) / 2;
    cnt[i] = count_less(keys + (int64_t)f * n, vals + (int64_t)f * n, n, mid);
  }
}
__global__ void split_update_kernel(int nbper, int nb, int P, int64_t n_global, unsigned long long* __restrict__ lohi,
                                   const unsigned long long* __restrict__ cnt) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nb; i += gridDim.x * blockDim.x) {
    const int b = i % nbper + 1;
    const unsigned long long t = (unsigned long long)(((__int128)b * n_global) / P);
    const unsigned long long lo = lohi[2 * i], hi = lohi[2 * i + 1];
    if (hi - lo <= 1) continue;
    const unsigned long long mid = lo + (hi - lo) / 2;
    if (cnt[i] <= t) lohi[2 * i] = mid;
    else lohi[2 * i + 1] = mid;
  }
}
// cut[f][q], q = 0..P: local entries of feature f below rank q's first key
__global__ void cut_kernel(const uint32_t* __restrict__ keys, const uint32_t* __restrict__ vals, int64_t n, int d,
                           int P, const unsigned long long* __restrict__ lohi, uint32_t* __restrict__ cut) {
  const int nbper = P - 1;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < d * (P + 1); i += gridDim.x * blockDim.x) {
    const int f = i / (P + 1), q = i % (P + 1);
    uint32_t c;
    if (q == 0) c = 0;
    else if (q == P) c = (uint32_t)n;
    else c = count_less(keys + (int64_t)f * n, vals + (int64_t)f * n, n, lohi[2 * (f * nbper + q - 1)]);
    cut[i] = c;
  }
}
// send[soff[f][q] + (i - cut[f][q])] = entry i of feature f's sorted list, q its destination
__global__ void pack_kernel(const uint32_t* __restrict__ keys, const uint32_t* __restrict__ vals,
                            const double* __restrict__ y, int64_t row0, int64_t n, int d, int P,
                            const uint32_t* __restrict__ cut, const unsigned long long* __restrict__ soff,
                            Sent* __restrict__ send) {
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n * d; t += (int64_t)gridDim.x * blockDim.x) {
    const int f = (int)(t / n);
    const uint32_t i = (uint32_t)(t - (int64_t)f * n);
    int q = 0;
    while (q + 1 < P && i >= cut[f * (P + 1) + q + 1]) ++q;
    Sent e;
    e.key = keys[t];
    e.row = vals[t];
    e.y = __ldg(y + (e.row - row0));
    send[soff[f * P + q] + (i - cut[f * (P + 1) + q])] = e;
  }
}
// received entry r (from rank q, feature f, index i) -> the concatenation of feature f's
// runs in source-rank order: keys / positions for the local stable sort
__global__ void unpack_kernel(const Sent* __restrict__ recv, int64_t nrecv, int d, int P,
                              const unsigned long long* __restrict__ roff, const unsigned long long* __restrict__ cpos,
                              uint32_t* __restrict__ keys, uint32_t* __restrict__ vals) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < nrecv; r += (int64_t)gridDim.x * blockDim.x) {
    int k = 0;  // largest (q, f) block with roff <= r (blocks in q-major, f-minor order)
    int lo = 0, hi = P * d;
    while (hi - lo > 1) {
      const int mid = (lo + hi) >> 1;
      if (roff[mid] <= (unsigned long long)r) lo = mid;
      else hi = mid;
    }
    k = lo;
    const int q = k / d, f = k % d;
    const unsigned long long pos = cpos[f * P + q] + ((unsigned long long)r - roff[k]);
    keys[pos] = recv[r].key;
    vals[pos] = (uint32_t)r;
  }
}
__global__ void __launch_bounds__(256) build_recv_kernel(const uint32_t* __restrict__ keys, const uint32_t* __restrict__ idx,
                                                         const Sent* __restrict__ recv, int64_t total,
                                                         float* __restrict__ lx, uint32_t* __restrict__ lr,
                                                         double* __restrict__ ly, const Ctl* ctl) {
  const bool y32 = ctl->y32 != 0;
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < total; p += (int64_t)gridDim.x * blockDim.x) {
    const Sent e = recv[idx[p]];
    lx[p] = unflip_f32(keys[p]);
    lr[p] = e.row;
    if (y32) reinterpret_cast<int32_t*>(ly)[p] = (int32_t)e.y;
    else ly[p] = e.y;
  }
}
// per feature list: the rank's boundary record (count, last x, sum of (y - c0)), fixed shape
__global__ void __launch_bounds__(256) root_bnd_kernel(const float* __restrict__ lx, const double* __restrict__ ly,
                                                       int64_t A0, const Ctl* __restrict__ ctl,
                                                       const NodeL* __restrict__ nodes0, BndRec* __restrict__ out) {
  const int f = blockIdx.x;
  const bool y32 = ctl->y32 != 0;
  const double c0 = nodes0[0].c;
  double acc = 0.0;
  for (int64_t i = threadIdx.x; i < A0; i += blockDim.x) {
    const int64_t p = (int64_t)f * A0 + i;
    const double yv = y32 ? (double)reinterpret_cast<const int32_t*>(ly)[p] : ly[p];
    acc = __dadd_rn(acc, __dsub_rn(yv, c0));
  }
  __shared__ double sh[256];
  sh[threadIdx.x] = acc;
  __syncthreads();
  for (int off = 128; off > 0; off >>= 1) {
    if (threadIdx.x < off) sh[threadIdx.x] = __dadd_rn(sh[threadIdx.x], sh[threadIdx.x + off]);
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    BndRec r;
    r.cnt = (uint32_t)A0;
    r.xlast = A0 ? lx[(int64_t)f * A0 + A0 - 1] : __int_as_float(0x7fc00000);
    r.s = sh[0];
    out[f] = r;
  }
}
// rank carries of the root's segments from the gathered records (rank order), the
// level-0 tables and the virtual-root plan
__global__ void __launch_bounds__(256) root_tables_sharded_kernel(Ctl* ctl, const NodeL* __restrict__ nodes0, int64_t A0,
                                                                  int d, int rank, int world,
                                                                  const BndRec* __restrict__ all, SegT* __restrict__ seg0,
                                                                  PSeg* __restrict__ pseg, uint32_t* __restrict__ desc0) {
  const NodeL rt = nodes0[0];
  const int64_t nch = (A0 * d + kChunkW - 1) / kChunkW;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nch; i += (int64_t)gridDim.x * blockDim.x)
    desc0[i] = (uint32_t)((i * kChunkW) / A0);
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    ctl->T[0] = (unsigned long long)A0 * d;
    ctl->T0[0] = (unsigned long long)A0;
  }
  for (int f = blockIdx.x * blockDim.x + threadIdx.x; f < d; f += gridDim.x * blockDim.x) {
    uint32_t ioff = 0;
    double soff = 0.0;
    float xprev = __int_as_float(0x7fc00000);
    for (int q = 0; q < rank; ++q) {
      const BndRec r = all[(int64_t)q * d + f];
      ioff += r.cnt;
      soff = __dadd_rn(soff, r.s);
      if (r.cnt) xprev = r.xlast;
    }
    SegT sg;
    sg.start = (uint64_t)f * (uint64_t)A0;
    sg.cnt = (uint32_t)A0;
    sg.k = 0;
    sg.f = f;
    sg.ioff = ioff;
    sg.soff = soff;
    sg.xprev = xprev;
    sg.pad = 0;
    seg0[f] = sg;
    PSeg p;
    p.start = sg.start;
    p.cnt = sg.cnt;
    p.k = 0;
    p.f = f;
    p.flags = PS_SPLIT | PS_ALLLEFT | (rt.searchable ? PS_SRCH0 : 0u);
    p.cs[0] = p.cs[1] = (uint32_t)f;
    p.ostart[0] = p.ostart[1] = sg.start;
    p.c[0] = p.c[1] = rt.c;
    p.v[0] = p.v[1] = rt.v;
    p.sc[0] = p.sc[1] = rt.sc;
    p.N[0] = p.N[1] = rt.N;
    p.ioff[0] = p.ioff[1] = ioff;
    p.soff[0] = p.soff[1] = soff;
    p.xprev[0] = p.xprev[1] = xprev;
    p.kid = 0;
    p.glim = 0;
    pseg[f] = p;
  }
  (void)world;
}

// Batched tile radix sort of the d lists of n (key, value) pairs (4 passes x 3 launches,
// stable).  Keys from b.k_in / b.v_in, or with X from the table itself (first pass,
// rows row0 + r).  Result in b.k_in / b.v_in, or with y straight in the level-0 lists
// (last pass).
void radix_sort_lists(const FitBufs& b, int64_t n, int d, cudaStream_t s, const float* X = nullptr,
                      int64_t row0 = 0, const double* y = nullptr) {
  uint32_t *ki = b.k_in, *ko = b.k_out, *vi = b.v_in, *vo = b.v_out;
  const int tiles = (int)((n + kTile - 1) / kTile);
  const unsigned g = (unsigned)(std::max(tiles, 1) * d);
  for (int pass = 0; pass < 4; ++pass) {
    const int shift = 8 * pass;
    const bool fx = X != nullptr && pass == 0, tl = y != nullptr && pass == 3;
    if (fx) rs_count_kernel<true><<<g, kTS, 0, s>>>(ki, X, n, d, shift, tiles, b.rs_cnt, b.ctl);
    else rs_count_kernel<false><<<g, kTS, 0, s>>>(ki, X, n, d, shift, tiles, b.rs_cnt, b.ctl);
    rs_offset_warp_kernel<<<(unsigned)((256 * d + 7) / 8), 256, 0, s>>>(b.rs_cnt, tiles, 256 * d, b.rs_off,
                                                                         b.rs_tot);
    RsOut o{ko, vo, b.lx[0], b.lr[0], b.ly[0], y, row0, b.ctl};
    if (fx) rs_scatter_kernel<true, false><<<g, kSTS, 0, s>>>(ki, vi, X, d, o, n, shift, tiles, b.rs_off, b.rs_tot);
    else if (tl) rs_scatter_kernel<false, true><<<g, kSTS, 0, s>>>(ki, vi, X, d, o, n, shift, tiles, b.rs_off, b.rs_tot);
    else rs_scatter_kernel<false, false><<<g, kSTS, 0, s>>>(ki, vi, X, d, o, n, shift, tiles, b.rs_off, b.rs_tot);
    std::swap(ki, ko);
    std::swap(vi, vo);
  }
}

}  // namespace

// Root statistics + presort of one rank's rows (P = 1: all rows) into the level-0 lists,
// plus the level-0 tables and the virtual-root plan.  X: n x d (row stride d), rows
// row0 .. row0 + n - 1 of the global table (their ids in the lists).
dt_status presort_enqueue(const FitBufs& b, const float* X, const double* y, int64_t n, int d, int dg,
                          int64_t row0, int32_t max_depth, int64_t min_leaf, cudaStream_t s) {
  (void)dg;
  const int64_t total0 = n * (int64_t)d;
  Ctl* ctl = b.ctl;
  {
    const int pr = prof_begin(PK_ROOT, s, 4);
    root_reduce_kernel<<<(unsigned)b.root_np, 256, 0, s>>>(y, n, b.root_chunk, reinterpret_cast<RootPart*>(b.parts));
    root_finalize_kernel<<<1, 256, 0, s>>>(reinterpret_cast<RootPart*>(b.parts), (int)b.root_np, n, ctl);
    root_center_kernel<<<(unsigned)b.root_np, 256, 0, s>>>(y, n, n, b.root_chunk, ctl, b.cparts);
    root_init_kernel<<<1, 256, 0, s>>>(b.cparts, (int)b.root_np, n, d, max_depth, min_leaf, ctl, b.nodes[0],
                                      b.dec_root);
    prof_end(pr, s, 16.0 * (double)n);  // y read twice
    DT_CK(cudaGetLastError());
  }
  {
    // the sort reads X in its first pass (keys, non-finite check) and writes the level-0
    // lists (x, row, y gathered) in its last
    int pr = prof_begin(PK_PRESORT_SORT, s, 12);
    radix_sort_lists(b, n, d, s, X, row0, y);
    prof_end(pr, s, 4.0 * 24.0 * (double)total0);  // per pass: keys read twice, pairs read + written
    DT_CK(cudaGetLastError());
    pr = prof_begin(PK_PRESORT_BUILD, s, 1);
    root_tables_kernel<<<num_sms(), 256, 0, s>>>(ctl, b.nodes[0], n, d, b.segs[0], b.pseg, b.desc[0]);
    prof_end(pr, s, 0.0);
    DT_CK(cudaGetLastError());
  }
  return DT_OK;
}

}  // namespace dtl

namespace dtl {

// Value-range sharded presort (see "value-range sharding" above) and the root.  X_local:
// n_local x d rows row0 .. row0 + n_local - 1 of the global table (rank order: row0 =
// rows of the lower ranks).  On return the level-0 lists hold this rank's A0 entries of
// every feature (global positions [p n / P, (p + 1) n / P)), with the rank carries.
dt_status presort_sharded_enqueue(const FitBufs& b, dt_comm* comm, const float* X, const double* y, int64_t n_local,
                                  int64_t row0, int64_t n_global, int d, int32_t max_depth, int64_t min_leaf,
                                  cudaStream_t s) {
  const int P = comm_world(comm), p = comm_rank(comm);
  const int64_t lo_p = (int64_t)(((__int128)p * n_global) / P), hi_p = (int64_t)(((__int128)(p + 1) * n_global) / P);
  const int64_t A0 = hi_p - lo_p;
  Ctl* ctl = b.ctl;
  std::vector<void*> tmp;
  auto alloc = [&](auto** ptr, size_t bytes) -> cudaError_t {
    cudaError_t e = cudaMallocAsync((void**)ptr, bytes ? bytes : 16, s);
    if (e == cudaSuccess) tmp.push_back((void*)*ptr);
    return e;
  };
  struct Free {
    std::vector<void*>& v;
    cudaStream_t s;
    ~Free() {
      for (void* q : v) cudaFreeAsync(q, s);
    }
  } freer{tmp, s};
  // ---- root statistics: per-rank partials, combined in rank order
  RootPart *mine = nullptr, *allp = nullptr;
  double *cmine = nullptr, *call = nullptr;
  DT_CK(alloc(&mine, sizeof(RootPart)));
  DT_CK(alloc(&allp, sizeof(RootPart) * P));
  DT_CK(alloc(&cmine, sizeof(double)));
  DT_CK(alloc(&call, sizeof(double) * P));
  const int npl = n_local > 0 ? (int)b.root_np : 0;
  int pr = prof_begin(PK_ROOT, s, 6);
  if (npl) root_reduce_kernel<<<npl, 256, 0, s>>>(y, n_local, b.root_chunk, reinterpret_cast<RootPart*>(b.parts));
  root_fold_kernel<<<1, 256, 0, s>>>(reinterpret_cast<RootPart*>(b.parts), npl, mine);
  DT_CK(cudaGetLastError());
  dt_status st = comm_allgather(comm, mine, allp, sizeof(RootPart), s);
  if (st != DT_OK) return st;
  root_finalize_kernel<<<1, 256, 0, s>>>(allp, P, n_global, ctl);
  if (npl) root_center_kernel<<<npl, 256, 0, s>>>(y, n_local, n_global, b.root_chunk, ctl, b.cparts);
  center_fold_kernel<<<1, 256, 0, s>>>(b.cparts, npl, cmine);
  DT_CK(cudaGetLastError());
  st = comm_allgather(comm, cmine, call, sizeof(double), s);
  if (st != DT_OK) return st;
  root_init_kernel<<<1, 256, 0, s>>>(call, P, n_global, d, max_depth, min_leaf, ctl, b.nodes[0], b.dec_root);
  prof_end(pr, s, 16.0 * (double)n_local);
  DT_CK(cudaGetLastError());
  // ---- local keys, local sort
  pr = prof_begin(PK_PRESORT_SORT, s, 14);
  if (n_local > 0) {
    radix_sort_lists(b, n_local, d, s, X, row0);
    DT_CK(cudaGetLastError());
  }
  // ---- exact splitters: 64 bisection rounds on the composite key, counts summed over ranks
  const int nbper = P - 1, nb = d * nbper;
  unsigned long long *lohi = nullptr, *cnt = nullptr;
  DT_CK(alloc(&lohi, sizeof(unsigned long long) * 2 * std::max(nb, 1)));
  DT_CK(alloc(&cnt, sizeof(unsigned long long) * std::max(nb, 1)));
  if (nb > 0) {
    split_init_kernel<<<1, 256, 0, s>>>(lohi, nb);
    for (int round = 0; round < 64; ++round) {
      split_count_kernel<<<(nb + 255) / 256, 256, 0, s>>>(b.k_in, b.v_in, n_local, nbper, nb, lohi, cnt);
      st = comm_allreduce_sum_u64(comm, cnt, nb, s);
      if (st != DT_OK) return st;
      split_update_kernel<<<(nb + 255) / 256, 256, 0, s>>>(nbper, nb, P, n_global, lohi, cnt);
    }
    DT_CK(cudaGetLastError());
  }
  uint32_t *cut = nullptr, *allcnt = nullptr;
  DT_CK(alloc(&cut, sizeof(uint32_t) * d * (P + 1)));
  DT_CK(alloc(&allcnt, sizeof(uint32_t) * d * P * P));
  cut_kernel<<<std::max(1, (d * (P + 1) + 255) / 256), 256, 0, s>>>(b.k_in, b.v_in, n_local, d, P, lohi, cut);
  DT_CK(cudaGetLastError());
  std::vector<uint32_t> hcut((size_t)d * (P + 1));
  DT_CK(cudaMemcpyAsync(hcut.data(), cut, sizeof(uint32_t) * hcut.size(), cudaMemcpyDeviceToHost, s));
  DT_CK(cudaStreamSynchronize(s));
  std::vector<uint32_t> mycnt((size_t)d * P);  // [f][q]
  for (int f = 0; f < d; ++f)
    for (int q = 0; q < P; ++q) mycnt[(size_t)f * P + q] = hcut[(size_t)f * (P + 1) + q + 1] - hcut[(size_t)f * (P + 1) + q];
  uint32_t* dmy = nullptr;
  DT_CK(alloc(&dmy, sizeof(uint32_t) * d * P));
  DT_CK(cudaMemcpyAsync(dmy, mycnt.data(), sizeof(uint32_t) * mycnt.size(), cudaMemcpyHostToDevice, s));
  st = comm_allgather(comm, dmy, allcnt, sizeof(uint32_t) * d * P, s);
  if (st != DT_OK) return st;
  std::vector<uint32_t> hall((size_t)d * P * P);  // [r][f][q]: rank r sends cnt entries of f to q
  DT_CK(cudaMemcpyAsync(hall.data(), allcnt, sizeof(uint32_t) * hall.size(), cudaMemcpyDeviceToHost, s));
  DT_CK(cudaStreamSynchronize(s));
  auto C = [&](int r, int f, int q) -> uint64_t { return hall[((size_t)r * d + f) * P + q]; };
  // ---- all-to-all of the entries: to rank q, feature after feature
  std::vector<size_t> scount(P), sdispl(P), rcount(P), rdispl(P);
  std::vector<unsigned long long> soff((size_t)d * P), roff((size_t)P * d), cpos((size_t)d * P);
  size_t sacc = 0, racc = 0;
  for (int q = 0; q < P; ++q) {
    sdispl[q] = sacc * sizeof(Sent);
    for (int f = 0; f < d; ++f) {
      soff[(size_t)f * P + q] = sacc;
      sacc += C(p, f, q);
    }
    scount[q] = sacc * sizeof(Sent) - sdispl[q];
    rdispl[q] = racc * sizeof(Sent);
    for (int f = 0; f < d; ++f) {
      roff[(size_t)q * d + f] = racc;
      racc += C(q, f, p);
    }
    rcount[q] = racc * sizeof(Sent) - rdispl[q];
  }
  if ((int64_t)racc != A0 * d) return fail(DT_ERR_CUDA, "dt_fit_sharded: splitters do not partition the positions");
  for (int f = 0; f < d; ++f) {
    unsigned long long acc = (unsigned long long)f * A0;
    for (int q = 0; q < P; ++q) {
      cpos[(size_t)f * P + q] = acc;
      acc += C(q, f, p);
    }
  }
  Sent *sendb = nullptr, *recvb = nullptr;
  unsigned long long *dsoff = nullptr, *droff = nullptr, *dcpos = nullptr;
  DT_CK(alloc(&sendb, sizeof(Sent) * (size_t)n_local * d));
  DT_CK(alloc(&recvb, sizeof(Sent) * (size_t)A0 * d));
  DT_CK(alloc(&dsoff, sizeof(unsigned long long) * soff.size()));
  DT_CK(alloc(&droff, sizeof(unsigned long long) * roff.size()));
  DT_CK(alloc(&dcpos, sizeof(unsigned long long) * cpos.size()));
  DT_CK(cudaMemcpyAsync(dsoff, soff.data(), sizeof(unsigned long long) * soff.size(), cudaMemcpyHostToDevice, s));
  DT_CK(cudaMemcpyAsync(droff, roff.data(), sizeof(unsigned long long) * roff.size(), cudaMemcpyHostToDevice, s));
  DT_CK(cudaMemcpyAsync(dcpos, cpos.data(), sizeof(unsigned long long) * cpos.size(), cudaMemcpyHostToDevice, s));
  const int gb = num_sms() * 8;
  if (n_local > 0) pack_kernel<<<gb, 256, 0, s>>>(b.k_in, b.v_in, y, row0, n_local, d, P, cut, dsoff, sendb);
  DT_CK(cudaGetLastError());
  st = comm_alltoallv(comm, sendb, scount.data(), sdispl.data(), recvb, rcount.data(), rdispl.data(), s);
  if (st != DT_OK) return st;
  // ---- the received runs, concatenated per feature in source-rank order, stable-sorted
  if (A0 > 0) {
    unpack_kernel<<<gb, 256, 0, s>>>(recvb, A0 * d, d, P, droff, dcpos, b.k_in, b.v_in);
    radix_sort_lists(b, A0, d, s);
    build_recv_kernel<<<gb, 256, 0, s>>>(b.k_in, b.v_in, recvb, A0 * d, b.lx[0], b.lr[0], b.ly[0], ctl);
    DT_CK(cudaGetLastError());
  }
  prof_end(pr, s, 0.0);
  // ---- rank carries of the root's segments, level-0 tables, virtual-root plan
  BndRec *bmine = nullptr, *ball = nullptr;
  DT_CK(alloc(&bmine, sizeof(BndRec) * d));
  DT_CK(alloc(&ball, sizeof(BndRec) * d * P));
  root_bnd_kernel<<<d, 256, 0, s>>>(b.lx[0], b.ly[0], A0, ctl, b.nodes[0], bmine);
  DT_CK(cudaGetLastError());
  st = comm_allgather(comm, bmine, ball, sizeof(BndRec) * d, s);
  if (st != DT_OK) return st;
  root_tables_sharded_kernel<<<num_sms(), 256, 0, s>>>(ctl, b.nodes[0], A0, d, p, P, ball, b.segs[0], b.pseg, b.desc[0]);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

}  // namespace dtl

namespace dtl {

namespace {

// Random Forest by expansion of the table's presorted lists: tree t's
// bootstrap sample has row r w_r times (w = the draw counts); its level-0 lists are the
// table's presorted lists with entry (x, r, y) repeated w_r times in place.  Equal x keep
// any order -- no split falls between equal x -- so integer-mode trees equal the exact
// CART of the sample in draw order (Reading R20); the copies keep row id r (they always go
// the same way).
__global__ void __launch_bounds__(256) boot_count_kernel(uint64_t seed, const uint32_t* __restrict__ tdev, int64_t n,
                                                         uint32_t* __restrict__ w, const double* __restrict__ y,
                                                         double* __restrict__ ys) {
  const uint32_t t = *tdev;  // the tree index lives on the device: one captured graph serves every tree
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t z = seed + 0x9E3779B97F4A7C15ull * ((((uint64_t)t) << 32) + (uint64_t)i + 1ull);  // Reading R21
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    z ^= z >> 31;
    const uint32_t r = (uint32_t)(z % (uint64_t)n);
    atomicAdd(w + r, 1u);
    ys[i] = __ldg(y + r);  // the sample's targets in draw order (root statistics)
  }
}

constexpr int kXT = 2048;  // entries per expansion tile
__global__ void __launch_bounds__(256) expand_sum_kernel(const uint32_t* __restrict__ lr, const uint32_t* __restrict__ w,
                                                         int64_t total, unsigned long long* __restrict__ tsum) {
  __shared__ unsigned long long sh[8];
  const int64_t base = (int64_t)blockIdx.x * kXT;
  unsigned long long acc = 0;
  for (int i = threadIdx.x; i < kXT; i += 256)
    if (base + i < total) acc += __ldg(w + __ldg(lr + base + i));
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t = 0;
    for (int q = 0; q < 8; ++q) t += sh[q];
    tsum[blockIdx.x] = t;
  }
}
__global__ void __launch_bounds__(1024) expand_scan_kernel(unsigned long long* __restrict__ tsum, int64_t ntiles) {
  __shared__ unsigned long long sh[33];
  __shared__ unsigned long long run;
  if (threadIdx.x == 0) run = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int64_t b0 = 0; b0 < ntiles; b0 += 1024) {
    const int64_t i = b0 + threadIdx.x;
    const unsigned long long v = i < ntiles ? tsum[i] : 0ull;
    unsigned long long inc = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const unsigned long long o = __shfl_up_sync(0xffffffffu, inc, d);
      if (lane >= d) inc += o;
    }
    if (lane == 31) sh[w] = inc;
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long r = 0;
      for (int q = 0; q < 32; ++q) { const unsigned long long t = sh[q]; sh[q] = r; r += t; }
      sh[32] = r;
    }
    __syncthreads();
    if (i < ntiles) tsum[i] = run + sh[w] + inc - v;
    __syncthreads();
    if (threadIdx.x == 0) run += sh[32];
    __syncthreads();
  }
}
template <bool kY32>
__global__ void __launch_bounds__(256) expand_write_kernel(const float* __restrict__ sx, const uint32_t* __restrict__ sr,
                                                           const double* __restrict__ sy, const uint32_t* __restrict__ w,
                                                           int64_t total, const unsigned long long* __restrict__ toff,
                                                           float* __restrict__ ox, uint32_t* __restrict__ orow,
                                                           double* __restrict__ oy) {
  using YT = typename std::conditional<kY32, uint32_t, unsigned long long>::type;
  __shared__ unsigned long long sh[9];
  const int64_t base = (int64_t)blockIdx.x * kXT;
  const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5;
  // thread t owns entries base + 8 t .. base + 8 t + 7 (in order)
  uint32_t cnt[8];
  unsigned long long tot = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    const int64_t p = base + 8 * threadIdx.x + j;
    cnt[j] = p < total ? __ldg(w + __ldg(sr + p)) : 0u;
    tot += cnt[j];
  }
  unsigned long long inc = tot;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const unsigned long long o = __shfl_up_sync(0xffffffffu, inc, d);
    if (lane >= d) inc += o;
  }
  if (lane == 31) sh[wp] = inc;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long r = 0;
    for (int q = 0; q < 8; ++q) { const unsigned long long t = sh[q]; sh[q] = r; r += t; }
  }
  __syncthreads();
  unsigned long long pos = toff[blockIdx.x] + sh[wp] + inc - tot;
  const YT* ys = reinterpret_cast<const YT*>(sy);
  YT* yo = reinterpret_cast<YT*>(oy);
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    const int64_t p = base + 8 * threadIdx.x + j;
    if (cnt[j]) {
      const float x = sx[p];
      const uint32_t r = sr[p];
      const YT yv = ys[p];
      for (uint32_t c = 0; c < cnt[j]; ++c) {
        ox[pos + c] = x;
        orow[pos + c] = r;
        yo[pos + c] = yv;
      }
      pos += cnt[j];
    }
  }
}

__global__ void set_storage_kernel(Ctl* ctl, int y32) { ctl->y32 = y32; }

}  // namespace

// Bootstrap tree t of a forest: draw counts, the sample's level-0 lists by expansion of the
// table's presorted lists (sx, sr, sy: n entries per feature), the root of the sample (its
// statistics in draw order) and the level-0 tables.  scratch: w (n u32), ys (n f64),
// tsum (n d / kXT + 1 u64).  y32: the lists' y storage (the table's, Reading R24).
dt_status forest_tree_enqueue(const FitBufs& b, const float* sx, const uint32_t* sr, const double* sy,
                              const double* y, int64_t n, int d, int32_t max_depth, int64_t min_leaf, uint64_t seed,
                              const uint32_t* tdev, int y32, uint32_t* w, double* ys, unsigned long long* tsum,
                              cudaStream_t s) {
  const int64_t total = n * (int64_t)d;
  const int64_t ntiles = (total + kXT - 1) / kXT;
  DT_CK(cudaMemsetAsync(w, 0, sizeof(uint32_t) * (size_t)n, s));
  DT_CK(cudaMemsetAsync(b.ctl, 0, sizeof(Ctl), s));
  const int gb = std::max(1, std::min<int>((int)((n + 255) / 256), num_sms() * 8));
  int pr = prof_begin(PK_PRESORT_BUILD, s, 4);
  boot_count_kernel<<<gb, 256, 0, s>>>(seed, tdev, n, w, y, ys);
  expand_sum_kernel<<<(unsigned)ntiles, 256, 0, s>>>(sr, w, total, tsum);
  expand_scan_kernel<<<1, 1024, 0, s>>>(tsum, ntiles);
  if (y32) expand_write_kernel<true><<<(unsigned)ntiles, 256, 0, s>>>(sx, sr, sy, w, total, tsum, b.lx[0], b.lr[0], b.ly[0]);
  else expand_write_kernel<false><<<(unsigned)ntiles, 256, 0, s>>>(sx, sr, sy, w, total, tsum, b.lx[0], b.lr[0], b.ly[0]);
  prof_end(pr, s, (16.0 + 4.0) * (double)total * 2.0);
  DT_CK(cudaGetLastError());
  pr = prof_begin(PK_ROOT, s, 6);
  root_reduce_kernel<<<(unsigned)b.root_np, 256, 0, s>>>(ys, n, b.root_chunk, reinterpret_cast<RootPart*>(b.parts));
  root_finalize_kernel<<<1, 256, 0, s>>>(reinterpret_cast<RootPart*>(b.parts), (int)b.root_np, n, b.ctl);
  root_center_kernel<<<(unsigned)b.root_np, 256, 0, s>>>(ys, n, n, b.root_chunk, b.ctl, b.cparts);
  root_init_kernel<<<1, 256, 0, s>>>(b.cparts, (int)b.root_np, n, d, max_depth, min_leaf, b.ctl, b.nodes[0], b.dec_root);
  set_storage_kernel<<<1, 1, 0, s>>>(b.ctl, y32);  // the lists keep the table's y storage
  root_tables_kernel<<<num_sms(), 256, 0, s>>>(b.ctl, b.nodes[0], n, d, b.segs[0], b.pseg, b.desc[0]);
  prof_end(pr, s, 16.0 * (double)n);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

}  // namespace dtl
