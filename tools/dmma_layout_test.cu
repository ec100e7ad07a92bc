// Checks the mma.sync.m8n8k4.f64 fragment layout assumed by kb1_v2.cuh (A row=lane>>2 col=lane&3;
// B row=lane&3 col=lane>>2; C/D row=lane>>2 cols 2*(lane&3)+{0,1}) against a plain product.
#include <cstdio>
__global__ void k(const double *A, const double *B, double *D) {
  int l = threadIdx.x;
  double a = A[(l >> 2) * 4 + (l & 3)];
  double b = B[(l & 3) * 8 + (l >> 2)];
  double c0 = 0, c1 = 0;
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
  D[(l >> 2) * 8 + 2 * (l & 3)] = c0;
  D[(l >> 2) * 8 + 2 * (l & 3) + 1] = c1;
}
int main() {
  double hA[32], hB[32], hD[64], ref[64];
  for (int i = 0; i < 32; ++i) { hA[i] = 1 + i * 0.37; hB[i] = 2 - i * 0.11; }
  for (int m = 0; m < 8; ++m) for (int n = 0; n < 8; ++n) { double s = 0; for (int kk = 0; kk < 4; ++kk) s += hA[m * 4 + kk] * hB[kk * 8 + n]; ref[m * 8 + n] = s; }
  double *dA, *dB, *dD;
  cudaMalloc(&dA, 256); cudaMalloc(&dB, 256); cudaMalloc(&dD, 512);
  cudaMemcpy(dA, hA, 256, cudaMemcpyHostToDevice); cudaMemcpy(dB, hB, 256, cudaMemcpyHostToDevice);
  k<<<1, 32>>>(dA, dB, dD);
  cudaMemcpy(hD, dD, 512, cudaMemcpyDeviceToHost);
  double e = 0; for (int i = 0; i < 64; ++i) e = fmax(e, fabs(hD[i] - ref[i]));
  printf("{\"dmma_layout_max_err\": %.3e}\n", e);
  return e < 1e-12 ? 0 : 1;
}
