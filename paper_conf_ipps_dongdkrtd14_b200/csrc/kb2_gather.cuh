// KB2 — deterministic node gather of the zone-local F_z.1 into global kinematic DOFs, plus the global
// min dt.  Replaces the paper's kernel 8 assembly / MFEM local->global step.
//
// Each node sums its incident (zone, local node) entries in ascending zone id (reading R20): a fixed
// order, so results are bitwise reproducible — no unordered atomics (north_star: "deterministic").
#pragma once

__global__ void __launch_bounds__(256) kb2_gather(const double *__restrict__ Fz1, const int32_t *__restrict__ ptr,
                                                  const int32_t *__restrict__ ent, int64_t num_nodes, int dim,
                                                  int nk, double *__restrict__ out, const double *__restrict__ cta_dt,
                                                  int num_cta, double *__restrict__ dt_out) {
  __shared__ double red[32];
  if (blockIdx.x == gridDim.x - 1) {
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
  for (int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; n < num_nodes; n += (int64_t)gridDim.x * blockDim.x) {
    const int b = __ldg(ptr + n), e = __ldg(ptr + n + 1);
    double s0 = 0.0, s1 = 0.0, s2 = 0.0;
    for (int i = b; i < e; ++i) {
      const int64_t o = __ldg(ent + i);   // z*dim*nk + a
      s0 += __ldg(Fz1 + o);
      s1 += __ldg(Fz1 + o + nk);
      if (dim == 3) s2 += __ldg(Fz1 + o + 2 * nk);
    }
    out[n] = s0;
    out[num_nodes + n] = s1;
    if (dim == 3) out[2 * num_nodes + n] = s2;
  }
}
