// Private interface between the corner-force handle (blast_cf.cu) and the time integrator
// (integrator.cu).  Not part of the C ABI: C++ linkage, hidden from include/.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/blast_cf.h"

namespace blastcf {

// read-only view of a handle's geometry and device maps
struct HandleView {
  int dim, k, nk, nt, nq;
  int64_t Z, nn;
  cudaStream_t stream;
  int device;
  const int32_t *zone_nodes;   // [Z][nk]
  const int32_t *ptr, *ent;    // node -> (z * dim * nk + a) CSR, ascending zone id
  const double *tab;           // B[n][p], G[n][p], Phi[n][t], qwt[n]
  bool multi_rank;
};

int handle_view(const blast_cf *h, HandleView *out);

// blast_cf_eval plus the per-point S(q) = alpha sigma adj(J)^T ([Z][Nq][dim][dim], device) that the
// energy right-hand side F^T Vbar of the integrator needs (eq (5)).
int eval_with_S(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                double *out_Fdot1, double *out_FTv, double *out_dt_min, double *Sq);

// records `msg` as blast_cf_last_error() of the calling thread and returns `code`
int set_error(int code, const char *msg);

}  // namespace blastcf
