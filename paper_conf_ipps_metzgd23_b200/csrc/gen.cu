// Synthetic feature-table generator: rows shaped like the paper's
// dataset row d = (y, p, c_1..c_m, t) (Eq. 1) with trainable
// parameters t (Table I range), executed PTX instructions p and a
// PTX-category histogram, GPU descriptors (SMs, clocks, memory bandwidth,
// L2, memory, cores/SM), target = latency.  Counter-based, so
// any row range can be generated on any device; bit-identical to datagen/__init__.py
// (same counters, same IEEE operation sequence, no FMA, hand-written exp).
#include "dt_internal.cuh"

namespace dtl {

namespace {

constexpr uint64_t kG = 0x9E3779B97F4A7C15ull;
constexpr uint64_t kH = 0xD1B54A32D192ED03ull;
constexpr int S_ROWCNN = 1, S_ROWGPU = 2, S_ROWNOISE = 3, S_CNN = 4, S_GPU = 5;

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t hash64(uint64_t seed, int stream, uint64_t i, uint64_t k) {
  const uint64_t key = mix64(seed ^ ((uint64_t)stream << 56));
  return mix64(key + i * kG + k * kH);
}
__device__ __forceinline__ double uni(uint64_t seed, int stream, uint64_t i, uint64_t k) {
  return __dmul_rn((double)(hash64(seed, stream, i, k) >> 11), 0x1.0p-53);
}

__device__ __forceinline__ double exp_det(double x) {
  const double coef[15] = {0x1.0000000000000p+0, 0x1.0000000000000p+0, 0x1.0000000000000p-1,
                           0x1.5555555555555p-3, 0x1.5555555555555p-5, 0x1.1111111111111p-7,
                           0x1.6c16c16c16c17p-10, 0x1.a01a01a01a01ap-13, 0x1.a01a01a01a01ap-16,
                           0x1.71de3a556c734p-19, 0x1.27e4fb7789f5cp-22, 0x1.ae64567f544e4p-26,
                           0x1.1eed8eff8d898p-29, 0x1.6124613a86d09p-33, 0x1.93974a8c07c9dp-37};
  const double t = __dmul_rn(x, 0x1.71547652b82fep+0);
  const double k = floor(t);
  const double s = __dmul_rn(__dsub_rn(t, k), 0x1.62e42fefa39efp-1);
  double p = coef[14];
#pragma unroll
  for (int j = 13; j >= 0; --j) p = __dadd_rn(__dmul_rn(p, s), coef[j]);
  return ldexp(p, (int)k);
}

__device__ __forceinline__ double log_uniform(double u, double lo, double log_ratio) {
  return __dmul_rn(lo, exp_det(__dmul_rn(u, log_ratio)));
}

__device__ __forceinline__ double irwin_hall(uint64_t seed, int stream, uint64_t i, uint64_t k0) {
  double z = 0.0;
#pragma unroll
  for (int j = 0; j < 12; ++j) z = __dadd_rn(z, uni(seed, stream, i, k0 + j));
  z = __dsub_rn(z, 6.0);
  return fmin(fmax(z, -4.0), 4.0);
}

__constant__ double c_sides[10] = {224.0, 240.0, 260.0, 299.0, 300.0, 331.0, 380.0, 456.0, 528.0, 600.0};
__constant__ double c_memgb[11] = {4.0, 8.0, 11.0, 16.0, 24.0, 32.0, 48.0, 80.0, 96.0, 141.0, 192.0};

// Writes the d feature columns of one row (as f64, before f32 rounding) into col[].
template <bool kExtra>
__device__ __forceinline__ void row_cols(uint64_t seed, uint64_t cid, uint64_t gid, double* col) {
  // ---- CNN side
  const double t = log_uniform(uni(seed, S_CNN, cid, 0), 3.5e6, 0x1.65f5a09d51accp+2);
  const double side = c_sides[hash64(seed, S_CNN, cid, 1) % 10ull];
  const double z = irwin_hall(seed, S_CNN, cid, 2);
  const double ratio = __ddiv_rn(side, 224.0);
  const double p = __dmul_rn(__dmul_rn(t, __dmul_rn(ratio, ratio)),
                             exp_det(__dadd_rn(3.0, __dmul_rn(0.5, z))));
  constexpr int nh = kExtra ? 16 : 8;
  double w[nh];
  double wsum = 0.0;
#pragma unroll
  for (int j = 0; j < nh; ++j) {
    w[j] = __dadd_rn(uni(seed, S_CNN, cid, 20 + 2 * j), uni(seed, S_CNN, cid, 21 + 2 * j));
  }
#pragma unroll
  for (int j = 0; j < nh; ++j) wsum = __dadd_rn(wsum, w[j]);
  // ---- GPU side
  const double sms = __dadd_rn(5.0, floor(__dmul_rn(uni(seed, S_GPU, gid, 0), 156.0)));
  const double clk = __dadd_rn(1000.0, floor(__dmul_rn(uni(seed, S_GPU, gid, 1), 1001.0)));
  const double bw = log_uniform(uni(seed, S_GPU, gid, 2), 80.0, 0x1.26bb1bbb55516p+2);
  const double l2 = log_uniform(uni(seed, S_GPU, gid, 3), 1.0, 0x1.3687a9f1af2b1p+2);
  const double mem = c_memgb[hash64(seed, S_GPU, gid, 4) % 11ull];
  const double cps = ((hash64(seed, S_GPU, gid, 5) & 1ull) == 0) ? 64.0 : 128.0;
  col[0] = t;
  col[1] = p;
#pragma unroll
  for (int j = 0; j < 8; ++j) col[2 + j] = __dmul_rn(p, __ddiv_rn(w[j], wsum));
  col[10] = sms;
  col[11] = clk;
  col[12] = bw;
  col[13] = l2;
  col[14] = mem;
  col[15] = cps;
  if (kExtra) {
    const double layers = floor(__dadd_rn(8.0, __dmul_rn(uni(seed, S_CNN, cid, 60), 1034.0)));
    const double neurons = log_uniform(uni(seed, S_CNN, cid, 61), 6.5e5, 0x1.d8c9fce2f10d0p+2);
    const double boost = __dadd_rn(clk, floor(__dmul_rn(uni(seed, S_GPU, gid, 6), 500.0)));
    const double regs = ((hash64(seed, S_GPU, gid, 7) & 1ull) == 0) ? 65536.0 : 131072.0;
    const double smem = __dadd_rn(64.0, floor(__dmul_rn(uni(seed, S_GPU, gid, 8), 165.0)));
    const double tdp = __dadd_rn(50.0, floor(__dmul_rn(uni(seed, S_GPU, gid, 9), 951.0)));
    const double tflops = __dmul_rn(__dmul_rn(__dmul_rn(__dmul_rn(sms, cps), 2.0), boost), 1e-6);
    col[16] = layers;
    col[17] = neurons;
    col[18] = side;
#pragma unroll
    for (int j = 8; j < 16; ++j) col[11 + j] = __dmul_rn(p, __ddiv_rn(w[j], wsum));
    col[27] = boost;
    col[28] = regs;
    col[29] = smem;
    col[30] = tdp;
    col[31] = tflops;
  }
}

template <bool kExtra>
__global__ void __launch_bounds__(128)
gen_table_kernel(uint64_t seed, int64_t row0, int64_t n, int real, uint64_t cmask, uint64_t gmask,
                 double unit_us, float* __restrict__ X, double* __restrict__ y) {
  constexpr int d = kExtra ? 32 : 16;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t row = (uint64_t)(row0 + i);
    const uint64_t cid = hash64(seed, S_ROWCNN, row, 0) & cmask;
    const uint64_t gid = hash64(seed, S_ROWGPU, row, 0) & gmask;
    double col[d];
    row_cols<kExtra>(seed, cid, gid, col);
    float xf[d];
#pragma unroll
    for (int j = 0; j < d; ++j) xf[j] = __double2float_rn(col[j]);
    float4* dst = reinterpret_cast<float4*>(X + i * d);
#pragma unroll
    for (int j = 0; j < d / 4; ++j) dst[j] = make_float4(xf[4 * j], xf[4 * j + 1], xf[4 * j + 2], xf[4 * j + 3]);
    if (y) {
      // target from the f32 features (datagen.latency_target)
      const double tt = (double)xf[0], pp = (double)xf[1];
      const double sms = (double)xf[10], clk = (double)xf[11], bw = (double)xf[12];
      const double compute = __ddiv_rn(pp, __dmul_rn(__dmul_rn(__dmul_rn(sms, clk), 1e6), 4.0));
      const double memory = __ddiv_rn(__dmul_rn(4.0, tt), __dmul_rn(bw, 1e9));
      const double zn = irwin_hall(seed, S_ROWNOISE, row, 0);
      const double lat = __dmul_rn(fmax(compute, memory), __dadd_rn(1.0, __dmul_rn(0.05, zn)));
      const double v = __ddiv_rn(__dmul_rn(lat, 1e6), unit_us);
      y[i] = real ? v : ceil(v);
    }
  }
}

__global__ void __launch_bounds__(128)
gen_dse_kernel(uint64_t seed, int64_t row0, int64_t n, int gbits, float* __restrict__ X) {
  const uint64_t gmask = (1ull << gbits) - 1ull;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t row = (uint64_t)(row0 + i);
    double col[16];
    row_cols<false>(seed, row >> gbits, row & gmask, col);
    float4* dst = reinterpret_cast<float4*>(X + i * 16);
#pragma unroll
    for (int j = 0; j < 4; ++j)
      dst[j] = make_float4(__double2float_rn(col[4 * j]), __double2float_rn(col[4 * j + 1]),
                           __double2float_rn(col[4 * j + 2]), __double2float_rn(col[4 * j + 3]));
  }
}

int gen_grid(int64_t n) {
  int64_t g = (n + 127) / 128;
  int64_t cap = (int64_t)num_sms() * 16;
  return (int)(g < cap ? (g < 1 ? 1 : g) : cap);
}

}  // namespace

dt_status gen_table_impl(uint64_t seed, int64_t row0, int64_t n, int32_t d, int32_t real,
                         int32_t cbits, int32_t gbits, double unit_us, float* X, double* y,
                         cudaStream_t s) {
  const uint64_t cm = (1ull << cbits) - 1ull, gm = (1ull << gbits) - 1ull;
  const int pr = prof_begin(PK_GEN, s, 1);
  if (d == 16)
    gen_table_kernel<false><<<gen_grid(n), 128, 0, s>>>(seed, row0, n, real, cm, gm, unit_us, X, y);
  else
    gen_table_kernel<true><<<gen_grid(n), 128, 0, s>>>(seed, row0, n, real, cm, gm, unit_us, X, y);
  prof_end(pr, s, (4.0 * d + (y ? 8.0 : 0.0)) * (double)n);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

dt_status gen_dse_impl(uint64_t seed, int64_t row0, int64_t n, int32_t gbits, float* X,
                       cudaStream_t s) {
  const int pr = prof_begin(PK_GEN, s, 1);
  gen_dse_kernel<<<gen_grid(n), 128, 0, s>>>(seed, row0, n, gbits, X);
  prof_end(pr, s, 64.0 * (double)n);
  DT_CK(cudaGetLastError());
  return DT_OK;
}

}  // namespace dtl
