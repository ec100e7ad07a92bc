// simultaneous H2D + D2H (two streams) vs one direction: is the e2e entry bound by PCIe duplex?
#include <cuda_runtime.h>
#include <cstdio>
int main() {
  const size_t up = 120u << 20, down = 68u << 20;
  char *hu, *hd, *du, *dd;
  cudaMallocHost(&hu, up); cudaMallocHost(&hd, down); cudaMalloc(&du, up); cudaMalloc(&dd, down);
  cudaStream_t s1, s2;
  cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
  cudaEvent_t a, b, c;
  cudaEventCreate(&a); cudaEventCreate(&b); cudaEventCreate(&c);
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(a, s1);
    cudaStreamWaitEvent(s2, a, 0);
    for (int i = 0; i < 8; ++i) cudaMemcpyAsync(du + i * (up / 8), hu + i * (up / 8), up / 8, cudaMemcpyHostToDevice, s1);
    for (int i = 0; i < 8; ++i) cudaMemcpyAsync(hd + i * (down / 8), dd + i * (down / 8), down / 8, cudaMemcpyDeviceToHost, s2);
    cudaEventRecord(b, s1);
    cudaEventRecord(c, s2);
    cudaEventSynchronize(b); cudaEventSynchronize(c);
    float m1, m2;
    cudaEventElapsedTime(&m1, a, b);
    cudaEventElapsedTime(&m2, a, c);
    printf("duplex: H2D 120 MB %.3f ms (%.1f GB/s), D2H 68 MB %.3f ms (%.1f GB/s)\n", m1, up / m1 / 1e6, m2, down / m2 / 1e6);
  }
  cudaEventRecord(a, s1);
  cudaMemcpyAsync(du, hu, up, cudaMemcpyHostToDevice, s1);
  cudaEventRecord(b, s1);
  cudaEventSynchronize(b);
  float m;
  cudaEventElapsedTime(&m, a, b);
  printf("H2D alone 120 MB %.3f ms (%.1f GB/s)\n", m, up / m / 1e6);
  return 0;
}
