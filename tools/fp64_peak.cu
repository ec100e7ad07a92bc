// FP64 peak microbenchmark for the roofline denominator.
// Measures on one B200: (1) DFMA throughput with independent FMA chains,
// (2) DMMA (mma.sync.m8n8k4.f64) throughput, (3) DSQRT/DDIV sequence cost.
// Prints one JSON line. Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_peak fp64_peak.cu
#include <cstdio>
#include <cuda_runtime.h>

#define CHECK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); return 1; } } while (0)

template <int CHAINS>
__global__ void dfma_kernel(double *out, int iters, double a, double b) {
  double acc[CHAINS];
#pragma unroll
  for (int c = 0; c < CHAINS; ++c) acc[c] = threadIdx.x * 1e-3 + c;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int c = 0; c < CHAINS; ++c) acc[c] = fma(acc[c], a, b);
  }
  double s = 0;
#pragma unroll
  for (int c = 0; c < CHAINS; ++c) s += acc[c];
  if (s == 12345.678) out[threadIdx.x] = s;
}

template <int ACC>
__global__ void dmma_kernel(double *out, int iters) {
  double a = 1.0 + threadIdx.x * 1e-6, b = 0.999;
  double c[ACC][2];
#pragma unroll
  for (int i = 0; i < ACC; ++i) { c[i][0] = 0; c[i][1] = 0; }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < ACC; ++i) {
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                   : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
    }
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < ACC; ++i) s += c[i][0] + c[i][1];
  if (s == 12345.678) out[threadIdx.x] = s;
}

__global__ void dsqrt_div_kernel(double *out, int iters) {
  double x = 1.0 + threadIdx.x * 1e-4, y = 2.0 + blockIdx.x * 1e-5;
  double z = 0.5, w = 0.25;
  for (int i = 0; i < iters; ++i) {
    x = sqrt(x + 1.0);
    y = 1.0 / (y + 0.5);
    z = sqrt(z + 2.0);
    w = 1.0 / (w + 1.5);
  }
  double s = x + y + z + w;
  if (s == 12345.678) out[threadIdx.x] = s;
}

int main() {
  int dev = 0;
  cudaDeviceProp prop;
  CHECK(cudaGetDeviceProperties(&prop, dev));
  int sms = prop.multiProcessorCount;
  double *out;
  CHECK(cudaMalloc(&out, 4096 * sizeof(double)));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float ms;

  // DFMA: 8 chains per thread, 512 threads, 4 blocks per SM
  const int iters = 20000;
  int blocks = sms * 4, threads = 512;
  for (int w = 0; w < 3; ++w) dfma_kernel<8><<<blocks, threads>>>(out, iters / 10, 0.999999, 1e-7);
  CHECK(cudaDeviceSynchronize());
  double best_dfma = 0;
  for (int r = 0; r < 10; ++r) {
    cudaEventRecord(e0);
    dfma_kernel<8><<<blocks, threads>>>(out, iters, 0.999999, 1e-7);
    cudaEventRecord(e1);
    CHECK(cudaEventSynchronize(e1));
    cudaEventElapsedTime(&ms, e0, e1);
    double tf = 2.0 * 8 * (double)iters * blocks * threads / (ms * 1e-3) / 1e12;
    if (tf > best_dfma) best_dfma = tf;
  }
  // sustained DFMA: back-to-back for ~3 s
  double sus_dfma = 0;
  {
    int reps = 0;
    cudaEventRecord(e0);
    for (; reps < 200; ++reps) dfma_kernel<8><<<blocks, threads>>>(out, iters, 0.999999, 1e-7);
    cudaEventRecord(e1);
    CHECK(cudaEventSynchronize(e1));
    cudaEventElapsedTime(&ms, e0, e1);
    sus_dfma = 2.0 * 8 * (double)iters * blocks * threads * reps / (ms * 1e-3) / 1e12;
  }

  // DMMA: 4 accumulators per warp
  const int mi = 20000;
  int mblocks = sms * 4, mthreads = 256;
  for (int w = 0; w < 3; ++w) dmma_kernel<4><<<mblocks, mthreads>>>(out, mi / 10);
  CHECK(cudaDeviceSynchronize());
  double best_dmma = 0;
  for (int r = 0; r < 10; ++r) {
    cudaEventRecord(e0);
    dmma_kernel<4><<<mblocks, mthreads>>>(out, mi);
    cudaEventRecord(e1);
    CHECK(cudaEventSynchronize(e1));
    cudaEventElapsedTime(&ms, e0, e1);
    double warps = (double)mblocks * mthreads / 32;
    double tf = 2.0 * 256 * 4 * (double)mi * warps / (ms * 1e-3) / 1e12;
    if (tf > best_dmma) best_dmma = tf;
  }

  // sqrt + div: 4 ops per iteration per thread (2 sqrt + 2 div)
  const int si = 4000;
  for (int w = 0; w < 2; ++w) dsqrt_div_kernel<<<blocks, threads>>>(out, si / 10);
  CHECK(cudaDeviceSynchronize());
  double best_sd = 0;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(e0);
    dsqrt_div_kernel<<<blocks, threads>>>(out, si);
    cudaEventRecord(e1);
    CHECK(cudaEventSynchronize(e1));
    cudaEventElapsedTime(&ms, e0, e1);
    double gops = 4.0 * si * (double)blocks * threads / (ms * 1e-3) / 1e9;
    if (gops > best_sd) best_sd = gops;
  }
  int clk_khz = 0;
  cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev);
  printf("{\"gpu\": \"%s\", \"sms\": %d, \"l2_bytes\": %d, \"smem_per_sm\": %zu, \"clock_khz_attr\": %d, "
         "\"dfma_tflops_burst\": %.3f, \"dfma_tflops_sustained\": %.3f, \"dmma_tflops_burst\": %.3f, "
         "\"sqrt_div_gops\": %.2f}\n",
         prop.name, sms, prop.l2CacheSize, prop.sharedMemPerMultiprocessor, clk_khz, best_dfma, sus_dfma,
         best_dmma, best_sd);
  return 0;
}
