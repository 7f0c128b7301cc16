// Root statistics and the presort of the exact CART fit (DESIGN.md
// "Kernels"): per-feature stable sort of (x, row id) once per fit, written as the level-0
// lists, the level-0 segment table, the chunk descriptors and the root node.
#include <algorithm>

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

__global__ void root_init_kernel(const double* parts, int nparts, int64_t n, int d, int32_t max_depth,
                                 int64_t min_leaf, Ctl* ctl, NodeL* nodes0, Decision* dec_root) {
  if (threadIdx.x != 0) return;
  double s = 0, cc = 0;
  for (int i = 0; i < nparts; ++i) neu_add(s, cc, parts[i]);
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
    p.pad = 0;
    pseg[f] = p;
  }
  (void)ctl;
}


// keys[f*n + r] = flip(x[r][f]); vals = row0 + r.  X row-major -> feature-major via smem.
__global__ void __launch_bounds__(256) presort_keys_kernel(const float* __restrict__ X, int64_t n, int d,
                                                           uint32_t* __restrict__ keys,
                                                           uint32_t* __restrict__ vals, Ctl* ctl, int64_t row0,
                                                           int rb) {
  extern __shared__ float tileX[];  // rb rows x d
  const int64_t r0 = (int64_t)blockIdx.x * rb;
  const int rows = (int)min((int64_t)rb, n - r0);
  const int64_t base = r0 * d;
  const int tot = rows * d;
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
      keys[(int64_t)f * n + r] = flip_f32(tileX[threadIdx.x * d + f]);
      vals[(int64_t)f * n + r] = (uint32_t)(row0 + r);
    }
  }
}

// SoA level-0 lists from the sorted pairs: x = unflip(key), row = val, y = y[row].
__global__ void __launch_bounds__(256) presort_build_kernel(const uint32_t* __restrict__ keys,
                                                            const uint32_t* __restrict__ vals,
                                                            const double* __restrict__ y, int64_t total,
                                                            float* __restrict__ lx, uint32_t* __restrict__ lr,
                                                            double* __restrict__ ly, const Ctl* ctl, int64_t row0) {
  const bool y32 = ctl->y32 != 0;
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < total;
       p += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t r = vals[p];
    lx[p] = unflip_f32(keys[p]);
    lr[p] = r;
    const double v = __ldg(y + (r - row0));
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
    root_finalize_kernel<<<1, 32, 0, s>>>(reinterpret_cast<RootPart*>(b.parts), (int)b.root_np, n, ctl);
    root_center_kernel<<<(unsigned)b.root_np, 256, 0, s>>>(y, n, b.root_chunk, ctl, b.cparts);
    root_init_kernel<<<1, 32, 0, s>>>(b.cparts, (int)b.root_np, n, d, max_depth, min_leaf, ctl, b.nodes[0],
                                      b.dec_root);
    prof_end(pr, s, 16.0 * (double)n);  // y read twice
    DT_CK(cudaGetLastError());
  }
  {
    const int rb = d <= 48 ? 256 : (d <= 96 ? 128 : 64);  // rows per block (smem)
    const int64_t nb = (n + rb - 1) / rb;
    const size_t smem = sizeof(float) * rb * (size_t)d;
    if (smem > 48 * 1024)
      DT_CK(cudaFuncSetAttribute(presort_keys_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int pr = prof_begin(PK_PRESORT_KEYS, s, 1);
    presort_keys_kernel<<<(unsigned)nb, 256, smem, s>>>(X, n, d, b.k_in, b.v_in, ctl, row0, rb);
    prof_end(pr, s, 16.0 * (double)total0);  // X read + (key, val) written
    DT_CK(cudaGetLastError());
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
    const int gb = std::max(1, std::min<int>((int)((total0 + 255) / 256), num_sms() * 8));
    pr = prof_begin(PK_PRESORT_BUILD, s, 2);
    presort_build_kernel<<<gb, 256, 0, s>>>(ki, vi, y, total0, b.lx[0], b.lr[0], b.ly[0], ctl, row0);
    root_tables_kernel<<<num_sms(), 256, 0, s>>>(ctl, b.nodes[0], n, d, b.segs[0], b.pseg, b.desc[0]);
    prof_end(pr, s, 36.0 * (double)total0);  // (key, val) read, y gathered, 16 B written
    DT_CK(cudaGetLastError());
  }
  return DT_OK;
}

}  // namespace dtl
