// PCIe copy probe: pinned H2D bandwidth vs copy size, 1D and 2D (3 rows of a [3][nn] array), back to back
#include <cuda_runtime.h>
#include <cstdio>
int main() {
  const size_t nn = 2146689, rowbytes = nn * 8;   // C4 node count: x is [3][nn]
  double *h, *d;
  cudaMallocHost(&h, 3 * rowbytes);
  cudaMalloc(&d, 3 * rowbytes);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (size_t kb : {256, 1024, 2048, 4096, 8192, 16384, 51200}) {
    const size_t bytes = kb * 1024, reps = (size_t)(3 * rowbytes) / bytes;
    for (int w = 0; w < 2; ++w) {
      cudaEventRecord(e0, s);
      for (size_t r = 0; r < reps; ++r) cudaMemcpyAsync((char *)d + r * bytes, (char *)h + r * bytes, bytes, cudaMemcpyHostToDevice, s);
      cudaEventRecord(e1, s);
      cudaEventSynchronize(e1);
    }
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    printf("1D %6zu KB x %4zu: %.1f GB/s (%.1f us per copy)\n", kb, reps, reps * bytes / (ms / 1e3) / 1e9, ms * 1e3 / reps);
  }
  for (size_t part : {8, 4, 2}) {   // 2D: the node range [0, nn/part) of all 3 rows in one call, part calls
    const size_t w = nn / part * 8;
    for (int ww = 0; ww < 2; ++ww) {
      cudaEventRecord(e0, s);
      for (size_t p = 0; p < part; ++p)
        cudaMemcpy2DAsync((char *)d + p * w, rowbytes, (char *)h + p * w, rowbytes, w, 3, cudaMemcpyHostToDevice, s);
      cudaEventRecord(e1, s);
      cudaEventSynchronize(e1);
    }
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    printf("2D 3 rows x %zu KB, %zu calls: %.1f GB/s\n", w / 1024, part, 3 * w * part / (ms / 1e3) / 1e9);
  }
  return 0;
}
