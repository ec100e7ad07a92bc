// Multi-GPU shared-DOF exchange (§3.4).
//
// BLAST/MFEM assemble zone contributions across MPI tasks through groups of shared DOFs with a master
// per group, and reduce the minimum time step with MPI.  Here: one process per B200,
// NCCL over NVLink.  After KB2 every rank holds its partial F.1 on the nodes it shares; it
//   1. packs them per neighbour (rows ordered by global node id, identical on both sides),
//   2. exchanges them with grouped ncclSend / ncclRecv on the handle's stream,
//   3. sums, for every shared node, the partials of all sharing ranks in ASCENDING RANK order, so every
//      sharer ends with bitwise identical values (reading R20),
// and takes the global min dt.  Two schedules:
//   overlap (zones numbered boundary-first): KB1 on the boundary zones; on a high-priority comm stream the
//     shared rows are gathered from the zone-local buffer and exchanged while KB1 runs on the interior
//     zones (on all but a few SMs, left to the pack and NCCL kernels); the dt allreduce(min) then overlaps
//     KB2; the ordered combine closes the eval;
//   single round (any numbering): KB1, KB2, then ONE grouped send/recv that carries each rank's dt next to
//     its F.1 rows (every rank of the block partitions neighbours every other, so no allreduce is needed;
//     otherwise an allreduce(min) follows).
// NCCL is loaded with dlopen at create time so that single-GPU use never touches it.
#pragma once
#include <dlfcn.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <vector>

#include "nccl.h"
#include "p2p.cuh"

namespace blastcf {

struct NcclApi {
  void *lib = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  ncclResult_t (*Send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  const char *(*GetErrorString)(ncclResult_t) = nullptr;
};

inline NcclApi *nccl_api() {
  static NcclApi api;
  static bool tried = false;
  if (tried) return api.lib ? &api : nullptr;
  tried = true;
  const char *cands[3] = {getenv("BLAST_CF_NCCL_LIB"), "libnccl.so.2", "libnccl.so"};
  for (const char *c : cands) {
    if (!c || !*c) continue;
    api.lib = dlopen(c, RTLD_NOW | RTLD_GLOBAL);
    if (api.lib) break;
  }
  if (!api.lib) return nullptr;
#define LOADSYM(field, name) api.field = (decltype(api.field))dlsym(api.lib, name)
  LOADSYM(GetUniqueId, "ncclGetUniqueId");
  LOADSYM(CommInitRank, "ncclCommInitRank");
  LOADSYM(CommDestroy, "ncclCommDestroy");
  LOADSYM(GroupStart, "ncclGroupStart");
  LOADSYM(GroupEnd, "ncclGroupEnd");
  LOADSYM(Send, "ncclSend");
  LOADSYM(Recv, "ncclRecv");
  LOADSYM(AllReduce, "ncclAllReduce");
  LOADSYM(GetErrorString, "ncclGetErrorString");
#undef LOADSYM
  if (!api.GetUniqueId || !api.CommInitRank || !api.Send || !api.Recv || !api.AllReduce || !api.GroupStart ||
      !api.GroupEnd || !api.CommDestroy) {
    api.lib = nullptr;
    return nullptr;
  }
  return &api;
}

inline int nccl_unique_id_bytes() { return (int)sizeof(ncclUniqueId); }

int nccl_fail(ncclResult_t r, const char *what);

// ---------------------------------------------------------------------------------------------
// Host plan (no CUDA): rows of the pack buffers and the ordered source list of every shared node.
// Row r of the send (and recv) buffer holds the dim partials of nbr_nodes[r] for neighbour i with
// nbr_offset[i] <= r < nbr_offset[i+1].  For each unique shared node u (ascending local id):
// sources src[src_ptr[u] .. src_ptr[u+1]) in ascending rank; src >= 0: own partial in send row src,
// src < 0: neighbour partial in recv row (-src - 1).
// ---------------------------------------------------------------------------------------------
struct ExchangePlan {
  std::vector<int32_t> unique_nodes;
  std::vector<int64_t> src_ptr, src;
};

inline ExchangePlan build_plan(int rank, int num_nbr, const int32_t *nbr_rank, const int64_t *nbr_offset,
                               const int32_t *nbr_nodes) {
  ExchangePlan pl;
  const int64_t total = num_nbr > 0 ? nbr_offset[num_nbr] : 0;
  // (node, rank, row) triples
  struct E { int32_t node, rank; int64_t row; };
  std::vector<E> es;
  es.reserve(total);
  for (int i = 0; i < num_nbr; ++i)
    for (int64_t r = nbr_offset[i]; r < nbr_offset[i + 1]; ++r) es.push_back({nbr_nodes[r], nbr_rank[i], r});
  std::sort(es.begin(), es.end(), [](const E &a, const E &b) {
    return a.node != b.node ? a.node < b.node : a.rank < b.rank;
  });
  pl.src_ptr.push_back(0);
  for (size_t i = 0; i < es.size();) {
    size_t j = i;
    while (j < es.size() && es[j].node == es[i].node) ++j;
    pl.unique_nodes.push_back(es[i].node);
    bool own_done = false;
    for (size_t t = i; t < j; ++t) {
      if (!own_done && rank < es[t].rank) { pl.src.push_back(es[i].row); own_done = true; }
      pl.src.push_back(-es[t].row - 1);
    }
    if (!own_done) pl.src.push_back(es[i].row);
    pl.src_ptr.push_back((int64_t)pl.src.size());
    i = j;
  }
  return pl;
}

// ---------------------------------------------------------------------------------------------
// device side
// ---------------------------------------------------------------------------------------------
__global__ void xch_pack(const double *__restrict__ F1, int64_t nn, int dim, const int32_t *__restrict__ rows,
                         int64_t nrows, double *__restrict__ send) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < nrows; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t node = rows[r];
    for (int c = 0; c < dim; ++c) send[r * dim + c] = F1[c * nn + node];
  }
}

__global__ void xch_combine(double *__restrict__ F1, int64_t nn, int dim, const int32_t *__restrict__ unodes,
                            int64_t nu, const int64_t *__restrict__ sptr, const int64_t *__restrict__ src,
                            const double *__restrict__ send, const double *__restrict__ recv) {
  for (int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; u < nu; u += (int64_t)gridDim.x * blockDim.x) {
    double s[3] = {0.0, 0.0, 0.0};
    for (int64_t i = sptr[u]; i < sptr[u + 1]; ++i) {
      const int64_t code = src[i];
      const double *row = code >= 0 ? send + code * dim : recv + (-code - 1) * dim;
#pragma unroll
      for (int c = 0; c < 3; ++c)   // (c < 3 unrolled: s stays in registers)
        if (c < dim) s[c] += row[c];
    }
    const int64_t node = unodes[u];
#pragma unroll
    for (int c = 0; c < 3; ++c)
      if (c < dim) F1[c * nn + node] = s[c];
  }
}

// Overlap schedule (boundary zones first): the partial F.1 of a shared row straight from the zone-local
// buffer, summed over the node's CSR entries in ascending zone id — the same order, hence the same bits,
// as KB2's gather of that node (every zone touching a shared node is a boundary zone).
__global__ void xch_pack_gather(const double *__restrict__ Fz1, const int32_t *__restrict__ ptr,
                                const int32_t *__restrict__ ent, int nk, int dim, const int32_t *__restrict__ rows,
                                int64_t nrows, double *__restrict__ send) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < nrows; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t node = rows[r];
    double s[3] = {0.0, 0.0, 0.0};
    for (int i = ptr[node]; i < ptr[node + 1]; ++i) {
      const int o = ent[i];
#pragma unroll
      for (int c = 0; c < 3; ++c)
        if (c < dim) s[c] += Fz1[o + c * nk];
    }
#pragma unroll
    for (int c = 0; c < 3; ++c)
      if (c < dim) send[r * dim + c] = s[c];
  }
}

// min over the per-CTA dt slots of this rank's corner-force launches (one block)
__global__ void xch_dt_reduce(const double *__restrict__ cta_dt, int n, double *__restrict__ out) {
  __shared__ double red[32];
  double m = __longlong_as_double(0x7ff0000000000000LL);
  for (int i = threadIdx.x; i < n; i += blockDim.x) m = fmin(m, cta_dt[i]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = fmin(m, __shfl_xor_sync(0xffffffffu, m, o));
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = m;
  __syncthreads();
  if (threadIdx.x < 32) {
    double r = threadIdx.x < (blockDim.x >> 5) ? red[threadIdx.x] : __longlong_as_double(0x7ff0000000000000LL);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) r = fmin(r, __shfl_xor_sync(0xffffffffu, r, o));
    if (threadIdx.x == 0) *out = r;
  }
}

// single-round schedule: dt = min(own, every neighbour's dt received with its F.1 rows)
__global__ void xch_dt_combine(double *__restrict__ dt, const double *__restrict__ recv_dt, int n) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    double m = *dt;
    for (int i = 0; i < n; ++i) m = fmin(m, recv_dt[i]);
    *dt = m;
  }
}

// peer-memory transport (p2p.cuh), set up by blast_cf_p2p_connect
struct P2PHost {
  void *mbox = nullptr;           // this rank's mailbox
  size_t mbox_bytes = 0;
  std::vector<void *> peer;       // mapped mailboxes of the other ranks (nullptr for this rank)
  std::vector<char> ipc_opened;   // 1: cudaIpcOpenMemHandle'd (closed at destroy)
  void *d_tab = nullptr;          // device tables of P2PDev (pointers, strides, counters)
  P2PDev dev{};
  uint64_t epoch = 0;             // evals run so far (the next one is epoch + 1)
  int send_blocks = 0, combine_blocks = 1;
  bool mapped = false;      // connect succeeded
  bool connected = false;   // eval uses this transport (blast_cf_p2p_enable can switch back to NCCL)
};

struct Exchange {
  NcclApi *api = nullptr;
  ncclComm_t comm = nullptr;
  int rank = 0, nranks = 1, dim = 0, num_nbr = 0;
  int64_t nn = 0, nrows = 0, nu = 0;
  std::vector<int32_t> nbr_rank;
  std::vector<int64_t> nbr_offset;
  std::vector<int32_t> h_rows;   // host copy of the shared-node rows (nbr_nodes)
  cudaStream_t stream = nullptr;
  int32_t *d_rows = nullptr, *d_unodes = nullptr;
  int64_t *d_sptr = nullptr, *d_src = nullptr;
  double *d_send = nullptr, *d_recv = nullptr, *d_tmp = nullptr;
  double *d_rdt = nullptr;       // [num_nbr] neighbours' dt (single-round schedule)
  // overlap schedule: zones [0, nb) touch shared nodes (boundary), [nb, Z) do not (interior)
  bool overlap = false;
  bool dt_piggy = false;   // single round: every rank neighbours every other, so the dt rides on the F.1 messages
  int64_t nb = 0;
  cudaStream_t s_comm = nullptr;   // high-priority stream of the pack / NCCL / dt work
  cudaEvent_t ev_s = nullptr, ev_b = nullptr, ev_i = nullptr, ev_p = nullptr, ev_x = nullptr, ev_sent = nullptr;
  P2PHost p2p;   // p2p.connected: eval moves the rows and dt through peer memory, no NCCL call
};

inline void exchange_destroy(Exchange *x) {
  if (!x) return;
  for (size_t t = 0; t < x->p2p.peer.size(); ++t)
    if (x->p2p.ipc_opened[t]) cudaIpcCloseMemHandle(x->p2p.peer[t]);
  cudaFree(x->p2p.mbox); cudaFree(x->p2p.d_tab);
  if (x->comm && x->api) x->api->CommDestroy(x->comm);
  cudaFree(x->d_rows); cudaFree(x->d_unodes); cudaFree(x->d_sptr); cudaFree(x->d_src);
  cudaFree(x->d_send); cudaFree(x->d_recv); cudaFree(x->d_tmp); cudaFree(x->d_rdt);
  for (cudaEvent_t e : {x->ev_s, x->ev_b, x->ev_i, x->ev_p, x->ev_x, x->ev_sent})
    if (e) cudaEventDestroy(e);
  if (x->s_comm) cudaStreamDestroy(x->s_comm);
  delete x;
}

// kernels of ours one eval launches besides KB1 / KB2 (NCCL's own kernels not counted)
inline int exchange_kernels(const Exchange *x) {
  if (x->p2p.connected)   // send rows (num_nbr > 0) + send dt + combine, plus the second KB1 launch of the overlap schedule
    return (x->overlap ? 1 : 0) + (x->num_nbr > 0 ? 1 : 0) + 2;
  const int combine = x->nu > 0 ? 1 : 0, pack = x->nrows > 0 ? 1 : 0;
  return x->overlap ? 1 /* second KB1 launch */ + pack + 1 /* dt reduce */ + combine : pack + combine + 1 /* dt combine */;
}

int exchange_create(Exchange **out, const blast_cf_mesh *mesh, int dim, int64_t nn, cudaStream_t stream,
                    const void *uid);
int exchange_allreduce_sum2(Exchange *x, double *a, double *b);
int exchange_run(Exchange *x, double *F1, double *dt);
int exchange_send_rows(Exchange *x, cudaStream_t st, bool with_dt, const double *dt);
void exchange_pack(Exchange *x, const double *F1);
void exchange_combine(Exchange *x, double *F1);
int nccl_get_unique_id(void *out);

}  // namespace blastcf
