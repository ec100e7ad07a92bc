// Peer-memory transport of the shared-DOF exchange (SURVEY §8(e) phase 2).
//
// The NCCL transport (exchange.cuh) packs the shared rows into a local buffer and hands them to
// ncclSend / ncclRecv, and reduces dt with ncclAllReduce.  Here the kernel that COMPUTES a shared row
// (the ordered sum of the node's zone-local F_z.1 entries, the same bits as KB2) STORES it straight into
// the neighbour's receive buffer over NVLink (CUDA IPC mapping of the peer's allocation), and signals
// with a system-scope release flag; the neighbour's combine kernel acquires the flags and sums the rows in
// ascending rank order.  The dt travels the same way (every rank writes its local dt into every other
// rank's slot), so no NCCL call is made per eval.
//
// Mailbox (one cudaMalloc per rank, zero-filled at connect; exported by cudaIpcGetMemHandle):
//   rows [2][nrows][dim]   recv rows, double-buffered by epoch parity; rows from rank r start at the
//                          receiver's nbr_offset of r (the same global-node order on both sides)
//   dt   [2][nranks]       every rank's local dt, by parity
//   flag_rows[nranks], flag_dt[nranks]   epoch of the rows / dt of rank r that have landed here
//   ack[nranks]            epoch up to which rank q has consumed what THIS rank sent it
// Eval number E (epoch, from 1) uses parity E & 1.  A sender writes parity p only after the receiver's
// ack >= E - 2 (the receiver has finished reading what E - 2 left there); the receiver acks after its
// combine.  No wait cycle: a combine waits only for sends, a send only for combines two evals back.
#pragma once
#include <cstdint>

namespace blastcf {

__device__ __forceinline__ uint64_t p2p_ld_acquire(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];\n" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void p2p_st_release(uint64_t *p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;\n" ::"l"(p), "l"(v) : "memory");
}
// spin until *p >= v; a peer that never arrives (dead process) traps after ~30 s instead of hanging
__device__ __forceinline__ void p2p_wait_geq(const uint64_t *p, uint64_t v) {
  const long long t0 = clock64();
  while (p2p_ld_acquire(p) < v) {
    __nanosleep(100);
    if (clock64() - t0 > (1LL << 36)) __trap();
  }
}

struct P2PDev {   // device-side view of the connected group (plain pointers, passed by value)
  // send side, per neighbour i (ascending rank): destination of rows [nbr_off[i], nbr_off[i+1]) in the
  // neighbour's mailbox (parity 0), the parity stride, the flag to release
  double *const *row_dst;
  const int64_t *row_pstride;
  uint64_t *const *row_flag;
  const int64_t *nbr_off;
  const int32_t *nbr_rank;
  const int32_t *blk_off;   // [num_nbr + 1] send blocks of neighbour i
  int32_t *cnt;             // [num_nbr] finished-block counters (self-resetting)
  int num_nbr;
  // dt, per rank t (t == me unused): slot base (parity 0) and flag in t's mailbox, the ack address in t's
  double *const *dt_dst;
  uint64_t *const *dt_flag;
  uint64_t *const *ack_dst;
  // this rank's own mailbox
  const double *rows;   // recv rows, parity 0
  int64_t rows_pstride;
  const double *dt;     // [2][nranks]
  const uint64_t *flag_rows, *flag_dt, *ack;
  int32_t *done;        // combine's finished-block counter
  int me, nranks;
};

// The shared rows of every neighbour, computed from the zone-local F_z.1 (ascending zone id, as KB2 and
// xch_pack_gather) and stored into the neighbour's mailbox; the last block of a neighbour releases its flag.
__global__ void p2p_send_rows(const double *__restrict__ Fz1, const int32_t *__restrict__ ptr,
                              const int32_t *__restrict__ ent, int nk, int dim, const int32_t *__restrict__ rows,
                              P2PDev g, uint64_t epoch) {
  int i = 0;
  while (i + 1 < g.num_nbr && (int)blockIdx.x >= g.blk_off[i + 1]) ++i;
  const int q = g.nbr_rank[i];
  if (threadIdx.x == 0 && epoch > 2) p2p_wait_geq(g.ack + q, epoch - 2);
  __syncthreads();
  const int nb = g.blk_off[i + 1] - g.blk_off[i], b = (int)blockIdx.x - g.blk_off[i];
  const int64_t r0 = g.nbr_off[i], r1 = g.nbr_off[i + 1];
  double *d = g.row_dst[i] + (epoch & 1) * g.row_pstride[i];
  for (int64_t r = r0 + (int64_t)b * blockDim.x + threadIdx.x; r < r1; r += (int64_t)nb * blockDim.x) {
    const int64_t node = rows[r];
    double s[3] = {0.0, 0.0, 0.0};
    for (int e = ptr[node]; e < ptr[node + 1]; ++e) {
      const int o = ent[e];
#pragma unroll
      for (int c = 0; c < 3; ++c)
        if (c < dim) s[c] += Fz1[o + c * nk];
    }
#pragma unroll
    for (int c = 0; c < 3; ++c)
      if (c < dim) __stcg(d + (r - r0) * dim + c, s[c]);
  }
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) {
    if (atomicAdd(g.cnt + i, 1) == nb - 1) {   // every block of this neighbour has written and fenced
      g.cnt[i] = 0;
      __threadfence_system();
      p2p_st_release(g.row_flag[i], epoch);
    }
  }
}

// This rank's dt (min over its per-CTA slots) to out_dt and into every other rank's mailbox (one block).
__global__ void p2p_send_dt(const double *__restrict__ cta_dt, int n, double *__restrict__ out_dt, P2PDev g,
                            uint64_t epoch) {
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
    if (threadIdx.x == 0) *out_dt = r;
    for (int t = threadIdx.x; t < g.nranks; t += 32) {
      if (t == g.me) continue;
      if (epoch > 2) p2p_wait_geq(g.ack + t, epoch - 2);
      __stcg(g.dt_dst[t] + (epoch & 1) * g.nranks + g.me, r);
      __threadfence_system();
      p2p_st_release(g.dt_flag[t], epoch);
    }
  }
}

// Ordered combine of the shared nodes (ascending rank: the plan of exchange.cuh, own partial = this rank's
// F.1 from KB2), the global min dt, then the acks (last block, after every block has read its rows).
__global__ void p2p_combine(double *__restrict__ F1, int64_t nn, int dim, const int32_t *__restrict__ unodes,
                            int64_t nu, const int64_t *__restrict__ sptr, const int64_t *__restrict__ src,
                            double *__restrict__ out_dt, P2PDev g, uint64_t epoch) {
  if (threadIdx.x == 0) {
    for (int i = 0; i < g.num_nbr; ++i) p2p_wait_geq(g.flag_rows + g.nbr_rank[i], epoch);
    if (blockIdx.x == 0)
      for (int t = 0; t < g.nranks; ++t)
        if (t != g.me) p2p_wait_geq(g.flag_dt + t, epoch);
    __threadfence_system();
  }
  __syncthreads();
  const double *recv = g.rows + (epoch & 1) * g.rows_pstride;
  for (int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; u < nu; u += (int64_t)gridDim.x * blockDim.x) {
    const int64_t node = unodes[u];
    double s[3] = {0.0, 0.0, 0.0};
    for (int64_t k = sptr[u]; k < sptr[u + 1]; ++k) {
      const int64_t code = src[k];
#pragma unroll
      for (int c = 0; c < 3; ++c)
        if (c < dim) s[c] += code >= 0 ? F1[c * nn + node] : __ldcg(recv + (-code - 1) * dim + c);
    }
#pragma unroll
    for (int c = 0; c < 3; ++c)
      if (c < dim) F1[c * nn + node] = s[c];
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    double m = *out_dt;
    const double *dts = g.dt + (epoch & 1) * g.nranks;
    for (int t = 0; t < g.nranks; ++t)
      if (t != g.me) m = fmin(m, __ldcg(dts + t));
    *out_dt = m;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(g.done, 1) == (int)gridDim.x - 1) {
      *g.done = 0;
      __threadfence_system();
      for (int t = 0; t < g.nranks; ++t)
        if (t != g.me) p2p_st_release(g.ack_dst[t], epoch);
    }
  }
}

}  // namespace blastcf
