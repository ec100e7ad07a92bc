// KB2 — deterministic node gather of the zone-local F_z.1 into global kinematic DOFs, plus the global
// min dt.  Replaces the paper's kernel 8 assembly / MFEM local->global step.
//
// Each node sums its incident (zone, local node) entries in ascending zone id (reading R20): a fixed
// order, so results are bitwise reproducible — no unordered atomics (north_star: "deterministic").
// One thread per node; the first MAXE entries' indices and values are all requested before any is
// summed (memory-level parallelism instead of a dependent load chain), nodes with more incident zones
// (unstructured meshes) finish in a loop.
#pragma once

// Nodes [n0, n1) of num_nodes (the host entry gathers node ranges as their zones complete); the last block
// also reduces the per-CTA dt slots when dt_out != nullptr.
template <int DIM, int MAXE>
__global__ void __launch_bounds__(256) kb2_gather(const double *__restrict__ Fz1, const int32_t *__restrict__ ptr,
                                                  const int32_t *__restrict__ ent, int64_t num_nodes, int64_t n0,
                                                  int64_t n1, int nk, double *__restrict__ out,
                                                  const double *__restrict__ cta_dt, int num_cta,
                                                  double *__restrict__ dt_out) {
  __shared__ double red[32];
  if (dt_out != nullptr && blockIdx.x == gridDim.x - 1) {
    double m = __longlong_as_double(0x7ff0000000000000LL);
    for (int i = threadIdx.x; i < num_cta; i += blockDim.x) m = fmin(m, cta_dt[i]);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = fmin(m, __shfl_xor_sync(0xffffffffu, m, o));
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = m;
    __syncthreads();
    if (threadIdx.x < 32) {
      double r = threadIdx.x < (blockDim.x >> 5) ? red[threadIdx.x] : __longlong_as_double(0x7ff0000000000000LL);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) r = fmin(r, __shfl_xor_sync(0xffffffffu, r, o));
      if (threadIdx.x == 0) *dt_out = r;
    }
  }
  const int64_t n = n0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= n1) return;
  const int b = __ldg(ptr + n), e = __ldg(ptr + n + 1);
  int o[MAXE];
#pragma unroll
  for (int i = 0; i < MAXE; ++i) o[i] = (b + i < e) ? __ldg(ent + b + i) : -1;
  double v[DIM][MAXE];
#pragma unroll
  for (int i = 0; i < MAXE; ++i)
#pragma unroll
    for (int c = 0; c < DIM; ++c) v[c][i] = o[i] >= 0 ? __ldg(Fz1 + o[i] + c * nk) : 0.0;
  double s[DIM];
#pragma unroll
  for (int c = 0; c < DIM; ++c) {
    s[c] = 0.0;
#pragma unroll
    for (int i = 0; i < MAXE; ++i)
      if (o[i] >= 0) s[c] += v[c][i];   // ascending zone id, the same order as the serial assembly
  }
  for (int i = b + MAXE; i < e; ++i) {
    const int oi = __ldg(ent + i);
#pragma unroll
    for (int c = 0; c < DIM; ++c) s[c] += __ldg(Fz1 + oi + c * nk);
  }
#pragma unroll
  for (int c = 0; c < DIM; ++c) out[c * num_nodes + n] = s[c];
}
