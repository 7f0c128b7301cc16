// Bandwidth probe for the scan's access pattern (not part of the library).
#include <cstdio>
#include <cuda_runtime.h>
template <int IT, bool DB>
__global__ void __launch_bounds__(256) rd(const float* __restrict__ x, const double* __restrict__ y, long total, double* out) {
  const long tile = 256L * IT;
  const long ntiles = (total + tile - 1) / tile;
  double acc = 0;
  float xn[IT]; double yn[IT];
  auto ld = [&](long t, float* xv, double* yv) {
    long p0 = t * tile + threadIdx.x * IT;
    const float4* x4 = (const float4*)(x + p0); const double2* y2 = (const double2*)(y + p0);
#pragma unroll
    for (int j = 0; j < IT / 4; ++j) { float4 v = __ldcs(x4 + j); xv[4*j]=v.x; xv[4*j+1]=v.y; xv[4*j+2]=v.z; xv[4*j+3]=v.w; }
#pragma unroll
    for (int j = 0; j < IT / 2; ++j) { double2 v = __ldcs(y2 + j); yv[2*j]=v.x; yv[2*j+1]=v.y; }
  };
  if (DB && blockIdx.x < ntiles) ld(blockIdx.x, xn, yn);
  for (long t = blockIdx.x; t < ntiles; t += gridDim.x) {
    float xv[IT]; double yv[IT];
    if (DB) {
#pragma unroll
      for (int j = 0; j < IT; ++j) { xv[j] = xn[j]; yv[j] = yn[j]; }
      if (t + gridDim.x < ntiles) ld(t + gridDim.x, xn, yn);
    } else ld(t, xv, yv);
#pragma unroll
    for (int j = 0; j < IT; ++j) acc += yv[j] * xv[j];
    __syncthreads();
  }
  if (acc == 12345.678) out[0] = acc;
}
template <int IT, bool DB>
void run(const float* x, const double* y, long total, double* o, int perSM) {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int grid = sms * perSM;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int w = 0; w < 3; ++w) rd<IT, DB><<<grid, 256>>>(x, y, total, o);
  cudaEventRecord(a);
  for (int r = 0; r < 20; ++r) rd<IT, DB><<<grid, 256>>>(x, y, total, o);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b); ms /= 20;
  printf("IT=%2d DB=%d perSM=%d grid=%d  %.1f us  %.0f GB/s\n", IT, (int)DB, perSM, grid, ms * 1e3, total * 12.0 / (ms * 1e-3) / 1e9);
}
int main() {
  long total = 16L << 20;
  float* x; double* y; double* o;
  cudaMalloc(&x, total * 4); cudaMalloc(&y, total * 8); cudaMalloc(&o, 8);
  cudaMemset(x, 0, total * 4); cudaMemset(y, 0, total * 8);
  for (int per : {1, 2, 3, 4, 8}) { run<8, false>(x, y, total, o, per); run<8, true>(x, y, total, o, per); run<16, false>(x, y, total, o, per); run<16, true>(x, y, total, o, per); }
  return 0;
}
