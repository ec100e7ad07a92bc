// Microbenchmark: do DFMA (CUDA-core FP64) and DMMA (mma.sync m8n8k4 f64) share a pipe on sm_100a?
// One CTA per SM, 16 warps: warps 0-7 run DFMA chains (CH independent chains per thread), warps 8-15 run
// DMMA chains (4 independent accumulators per warp).  mode 0 = DFMA warps only, 1 = DMMA warps only,
// 2 = both.  Prints per-group cycles per iteration.  Used to explain the KB1 v5 PW/KW interference.
#include <cstdio>
#include <cuda_runtime.h>

template <int CH>
__global__ void k(double *out, long long *cyc, int iters, int mode) {
  const int w = threadIdx.x >> 5;
  const bool is_f = w < 8;
  if ((is_f && mode == 1) || (!is_f && mode == 0)) return;
  long long t0 = clock64();
  double r = 0.0;
  if (is_f) {
    double acc[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) acc[c] = threadIdx.x + c;
    const double a = 0.999999, b = 1e-7;
    for (int i = 0; i < iters; ++i)
#pragma unroll
      for (int c = 0; c < CH; ++c) acc[c] = fma(acc[c], a, b);
#pragma unroll
    for (int c = 0; c < CH; ++c) r += acc[c];
  } else {
    double d[4][2];
#pragma unroll
    for (int c = 0; c < 4; ++c) d[c][0] = d[c][1] = 0.0;
    const double a = 1.0 + threadIdx.x * 1e-9, b = 0.5;
    for (int i = 0; i < iters / 8; ++i)
#pragma unroll
      for (int c = 0; c < 4; ++c)
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                     : "+d"(d[c][0]), "+d"(d[c][1]) : "d"(a), "d"(b));
#pragma unroll
    for (int c = 0; c < 4; ++c) r += d[c][0] + d[c][1];
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = r;
  if ((threadIdx.x & 31) == 0) cyc[blockIdx.x * 16 + w] = t1 - t0;
}

template <int CH>
void run(int sms, double *out, long long *cyc, long long *h) {
  const int iters = 1 << 16;
  for (int mode = 0; mode < 3; ++mode) {
    k<CH><<<sms, 512>>>(out, cyc, iters, mode);
    cudaDeviceSynchronize();
    cudaMemcpy(h, cyc, sizeof(long long) * sms * 16, cudaMemcpyDeviceToHost);
    double f = 0, m = 0;
    for (int b = 0; b < sms; ++b) {
      f += h[b * 16 + 0];
      m += h[b * 16 + 8];
    }
    f /= sms;
    m /= sms;
    // per SMSP: 2 DFMA warps x CH chains x iters DFMA; 2 DMMA warps x 4 x iters/8 DMMA
    printf("CH=%d mode=%d  DFMA warps: %.0f cyc (%.2f cyc/DFMA-warp-inst per SMSP)   DMMA warps: %.0f cyc (%.2f cyc/DMMA per SMSP)\n",
           CH, mode, mode == 1 ? 0.0 : f, mode == 1 ? 0.0 : f / (2.0 * CH * iters), mode == 0 ? 0.0 : m,
           mode == 0 ? 0.0 : m / (2.0 * 4 * (iters / 8)));
  }
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double *out;
  long long *cyc, *h = new long long[sms * 16];
  cudaMalloc(&out, sizeof(double) * sms * 512);
  cudaMalloc(&cyc, sizeof(long long) * sms * 16);
  run<1>(sms, out, cyc, h);
  run<2>(sms, out, cyc, h);
  run<4>(sms, out, cyc, h);
  run<8>(sms, out, cyc, h);
  return 0;
}
