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
  int rank, nranks;            // of the domain decomposition (0, 1 on one GPU)
  bool loopback;               // multi-rank handle of a one-device test group (no NCCL communicator)
};

int handle_view(const blast_cf *h, HandleView *out);

// ---- group communication of multi-rank solvers --------------------------------
// A "group" is the set of handles one call drives: n = 1 (this process's rank; the other ranks make
// the same call; NCCL moves the data) or, for tests on one GPU, all n ranks of a loopback group
// (device copies and an ascending-rank host reduction move the data).  Single-rank handles: no-ops.
// Every call is enqueued on / synchronizes with the handles' streams as needed; arrays are device.
//
// group_exchange_sum: shared-node sum of [dim][nn] vectors: every sharer ends with the sum of all
// sharers' values in ascending rank order (the F.1 exchange of blast_cf_eval, on another vector).
int group_exchange_sum(blast_cf *const *hs, int n, double *const *vec);
// group_allreduce: buf[r][0..count) of every rank replaced by the elementwise sum (op 0), min (1) or
// max (2) over all ranks; every rank gets bitwise the same values.
int group_allreduce(blast_cf *const *hs, int n, double *const *buf, int count, int op);
// owner weights of the local nodes: 1 where this rank is the lowest rank holding the node, else 0
// (shared-node dot products count each node once, as MFEM's group masters)
int owner_weights(const blast_cf *h, double *host_out);

// blast_cf_eval plus the per-point S(q) = alpha sigma adj(J)^T ([Z][Nq][dim][dim], device) that the
// energy right-hand side F^T Vbar of the integrator needs (eq (5)).
int eval_with_S(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                double *out_Fdot1, double *out_FTv, double *out_dt_min, double *Sq);

// records `msg` as blast_cf_last_error() of the calling thread and returns `code`
int set_error(int code, const char *msg);

}  // namespace blastcf
