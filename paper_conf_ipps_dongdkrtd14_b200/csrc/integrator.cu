// integrator.cu — the time step around the corner force (API in include/blast_cf.h).
//
// Momentum:  M_V dv/dt = -F.1   ("solved with PCG"; kernel 9, 405-413)
// Energy:    M_E de/dt = F^T v  (M_E^{-1} precomputed; kernel 11 "SpMV", 414-420)
// Position:  dx/dt = v
//
// B200 design:
//   * M_V is applied matrix-free: per zone u_z -> B (nodes -> quadrature points, sum factorization)
//     -> * alpha_q rho0|J0|(q) -> B^T, written zone-locally ([Z][dim][Nk], the KB1 output layout) and
//     gathered to the nodes in ascending zone id through the corner-force handle's CSR.  Bitwise
//     deterministic, no atomics, no assembled sparse matrix (an assembled 3D Q4 M_V would hold
//     ~200 nonzeros per row; its SpMV reads 10x the bytes of one zone pass).
//   * CG: Jacobi preconditioner, the dim component systems in lockstep, all scalars device-resident;
//     three kernels per iteration (zone action, gather + p.Ap, update + r.z), each ending with a
//     deterministic last-block reduction; converged kernels exit at entry; the host polls the
//     converged flag every `cg_check_every` iterations.
//   * F^T Vbar from the S(q) the corner-force kernel writes: grad Vbar at the points by sum
//     factorization, contracted with S, projected on phi_j (the KB1 back stage, one component).
//   * M_E^{-1}: tensor-product 1-D inverses when rho0|J0| is constant on the zone, else a dense per-zone
//     inverse built at create in long double.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <vector>

#include "internal.h"
#include "tables.h"

namespace {

using blastcf::HandleView;

int fail(int code, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  return blastcf::set_error(code, buf);
}

#define CUDA_TRY(expr)                                                                       \
  do {                                                                                       \
    cudaError_t e_ = (expr);                                                                 \
    if (e_ != cudaSuccess)                                                                   \
      return fail(e_ == cudaErrorMemoryAllocation ? BLAST_CF_ENOMEM : BLAST_CF_ECUDA,        \
                  "%s: %s (%s:%d)", #expr, cudaGetErrorString(e_), __FILE__, __LINE__);      \
  } while (0)

constexpr int ZT = 128;   // threads of the per-zone kernels
constexpr int NB = 256;   // threads of the per-node kernels

// device-resident CG scalars, one set per velocity component
struct CGScal {
  double rz[3], bb[3], alpha[3], beta[3], rr[3];
  double tol2;
  int done, iters;
  unsigned ticket;
};

// ------------------------------------------------------------------------------------------------
// sum-factorization building block: in[s2][s1][s0] -> out with axis AX (length s_AX) replaced by m,
//   out(.., o, ..) = sum_i M[o * ldo + i * ldi] in(.., i, ..)
// (ldo = p, ldi = 1 applies an [n][p] table forward; ldo = 1, ldi = p its transpose).  No barrier.
// ------------------------------------------------------------------------------------------------
template <int AX>
__device__ __forceinline__ void contract(const double *__restrict__ in, double *__restrict__ out, int s0, int s1,
                                         int s2, int m, const double *__restrict__ M, int ldo, int ldi) {
  const int e0 = AX == 0 ? m : s0, e1 = AX == 1 ? m : s1, e2 = AX == 2 ? m : s2;
  const int nin = AX == 0 ? s0 : AX == 1 ? s1 : s2;
  const int stride = AX == 0 ? 1 : AX == 1 ? s0 : s0 * s1;
  const int tot = e0 * e1 * e2;
  for (int idx = threadIdx.x; idx < tot; idx += blockDim.x) {
    const int i0 = idx % e0, i1 = (idx / e0) % e1, i2 = idx / (e0 * e1);
    const int o = AX == 0 ? i0 : AX == 1 ? i1 : i2;
    const int base = AX == 0 ? (i2 * s1 + i1) * s0 : AX == 1 ? i2 * s1 * s0 + i0 : i1 * s0 + i0;
    double acc = 0.0;
    for (int i = 0; i < nin; ++i) acc = fma(M[o * ldo + i * ldi], in[base + i * stride], acc);
    out[idx] = acc;
  }
}

// forward interpolation nodes [p]^D -> points [n]^D with the [n][p] table T (values B); a, b: buffers
// of >= n^D doubles; returns the buffer that holds the result
template <int D>
__device__ double *to_points(double *a, double *b, const double *T, int n, int p) {
  if (D == 2) {
    contract<0>(a, b, p, p, 1, n, T, p, 1); __syncthreads();
    contract<1>(b, a, n, p, 1, n, T, p, 1); __syncthreads();
    return a;
  }
  contract<0>(a, b, p, p, p, n, T, p, 1); __syncthreads();
  contract<1>(b, a, n, p, p, n, T, p, 1); __syncthreads();
  contract<2>(a, b, n, n, p, n, T, p, 1); __syncthreads();
  return b;
}

// back projection points [n]^D -> [m]^D with the transpose of an [n][m] table T
template <int D>
__device__ double *from_points(double *a, double *b, const double *T, int n, int m) {
  if (D == 2) {
    contract<0>(a, b, n, n, 1, m, T, 1, m); __syncthreads();
    contract<1>(b, a, m, n, 1, m, T, 1, m); __syncthreads();
    return a;
  }
  contract<0>(a, b, n, n, n, m, T, 1, m); __syncthreads();
  contract<1>(b, a, m, n, n, m, T, 1, m); __syncthreads();
  contract<2>(a, b, m, m, n, m, T, 1, m); __syncthreads();
  return b;
}

__device__ __forceinline__ int ipow(int b, int e) { int r = 1; for (int i = 0; i < e; ++i) r *= b; return r; }

// alpha_q rho0|J0|(z, q) for every point of zone z into wq[nq]
template <int D>
__device__ void zone_weights(double *wq, const double *w1, const double *R, int64_t z, int n) {
  const int nq = ipow(n, D);
  for (int q = threadIdx.x; q < nq; q += blockDim.x) {
    double a = w1[q % n] * w1[(q / n) % n];
    if (D == 3) a *= w1[q / (n * n)];
    wq[q] = a * R[z * nq + q];
  }
}

// ------------------------------------------------------------------------------------------------
// deterministic block / grid reductions (fixed shuffle tree, fixed warp order, fixed block order)
// ------------------------------------------------------------------------------------------------
template <int NC>
__device__ void block_sum(double (&v)[NC], double *red) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
#pragma unroll
  for (int c = 0; c < NC; ++c) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v[c] += __shfl_xor_sync(0xffffffffu, v[c], o);
    if (lane == 0) red[c * 32 + warp] = v[c];
  }
  __syncthreads();
  if (warp == 0) {
#pragma unroll
    for (int c = 0; c < NC; ++c) {
      double r = lane < nw ? red[c * 32 + lane] : 0.0;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) r += __shfl_xor_sync(0xffffffffu, r, o);
      v[c] = r;
    }
  }
  __syncthreads();
}

// block partials -> partials[blockIdx][NC]; the last block to arrive sums them in block order.
// Returns true in the last block; there thread 0 holds the grid totals in v.
template <int NC>
__device__ bool grid_sum(double (&v)[NC], double *partials, unsigned *ticket) {
  __shared__ double red[NC * 32];
  __shared__ bool last;
  block_sum<NC>(v, red);
  if (threadIdx.x == 0) {
#pragma unroll
    for (int c = 0; c < NC; ++c) partials[(size_t)blockIdx.x * NC + c] = v[c];
    __threadfence();
    last = atomicAdd(ticket, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!last) return false;
  __threadfence();
  double s[NC];
#pragma unroll
  for (int c = 0; c < NC; ++c) s[c] = 0.0;
  for (unsigned b = threadIdx.x; b < gridDim.x; b += blockDim.x)
#pragma unroll
    for (int c = 0; c < NC; ++c) s[c] += __ldcg(partials + (size_t)b * NC + c);
  block_sum<NC>(s, red);
#pragma unroll
  for (int c = 0; c < NC; ++c) v[c] = s[c];
  if (threadIdx.x == 0) *ticket = 0u;
  return true;
}

// ------------------------------------------------------------------------------------------------
// per-zone kernels (one CTA per zone)
// ------------------------------------------------------------------------------------------------
struct ZoneArgs {
  const double *tab;          // B[n][p], G[n][p], Phi[n][t], qwt[n]
  const int32_t *zone_nodes;  // [Z][nk]
  const double *R;            // rho0|J0| [Z][nq]
  int64_t Z, nn;
  int k;
};

// Y_z = M_z (u + beta P)_z per component (beta NULL: M_z u_z); kinematic mass action
template <int D>
__global__ void __launch_bounds__(ZT) k_mass_zone(ZoneArgs za, const double *__restrict__ u,
                                                  const double *__restrict__ Pold, const CGScal *sc,
                                                  double *__restrict__ Y) {
  if (sc && sc->done) return;
  extern __shared__ double sm[];
  const int k = za.k, n = 2 * k, p = k + 1, nk = ipow(p, D), nq = ipow(n, D);
  double *B = sm, *w1 = B + n * p, *wq = w1 + n, *b0 = wq + nq, *b1 = b0 + nq;
  for (int i = threadIdx.x; i < n * p; i += blockDim.x) B[i] = za.tab[i];
  for (int i = threadIdx.x; i < n; i += blockDim.x) w1[i] = za.tab[2 * n * p + n * k + i];
  __syncthreads();
  const int64_t z = blockIdx.x;
  zone_weights<D>(wq, w1, za.R, z, n);
  const int32_t *zn = za.zone_nodes + z * nk;
  for (int c = 0; c < D; ++c) {
    const double beta = sc ? sc->beta[c] : 0.0;
    for (int a = threadIdx.x; a < nk; a += blockDim.x) {
      const int64_t g = (int64_t)c * za.nn + zn[a];
      b0[a] = sc ? __fma_rn(beta, Pold[g], u[g]) : u[g];
    }
    __syncthreads();
    double *f = to_points<D>(b0, b1, B, n, p);
    for (int q = threadIdx.x; q < nq; q += blockDim.x) f[q] *= wq[q];
    __syncthreads();
    double *o = from_points<D>(f, f == b0 ? b1 : b0, B, n, p);
    for (int a = threadIdx.x; a < nk; a += blockDim.x) Y[(z * D + c) * nk + a] = o[a];
    __syncthreads();
  }
}

// diagonal of M_z (sum_q wq W_a(q)^2, via the squared table) into every component slot of Y_z
template <int D>
__global__ void __launch_bounds__(ZT) k_diag_zone(ZoneArgs za, double *__restrict__ Y) {
  extern __shared__ double sm[];
  const int k = za.k, n = 2 * k, p = k + 1, nk = ipow(p, D), nq = ipow(n, D);
  double *B2 = sm, *w1 = B2 + n * p, *b0 = w1 + n, *b1 = b0 + nq;
  for (int i = threadIdx.x; i < n * p; i += blockDim.x) B2[i] = za.tab[i] * za.tab[i];
  for (int i = threadIdx.x; i < n; i += blockDim.x) w1[i] = za.tab[2 * n * p + n * k + i];
  __syncthreads();
  const int64_t z = blockIdx.x;
  zone_weights<D>(b0, w1, za.R, z, n);
  __syncthreads();
  double *o = from_points<D>(b0, b1, B2, n, p);
  for (int a = threadIdx.x; a < nk; a += blockDim.x)
    for (int c = 0; c < D; ++c) Y[(z * D + c) * nk + a] = o[a];
}

// me1_z[j] = sum_q wq phi_j(q)   (row sums of M_E: the internal-energy weights)
template <int D>
__global__ void __launch_bounds__(ZT) k_me1_zone(ZoneArgs za, double *__restrict__ me1) {
  extern __shared__ double sm[];
  const int k = za.k, n = 2 * k, t = k, nt = ipow(t, D), nq = ipow(n, D);
  double *Phi = sm, *w1 = Phi + n * t, *b0 = w1 + n, *b1 = b0 + nq;
  for (int i = threadIdx.x; i < n * t; i += blockDim.x) Phi[i] = za.tab[2 * n * (k + 1) + i];
  for (int i = threadIdx.x; i < n; i += blockDim.x) w1[i] = za.tab[2 * n * (k + 1) + n * k + i];
  __syncthreads();
  const int64_t z = blockIdx.x;
  zone_weights<D>(b0, w1, za.R, z, n);
  __syncthreads();
  double *o = from_points<D>(b0, b1, Phi, n, t);
  for (int j = threadIdx.x; j < nt; j += blockDim.x) me1[z * nt + j] = o[j];
}

// de_z = M_E,z^{-1} F_z^T Vbar_z with (F_z^T Vbar_z)_j = sum_q phi_j(q) sum_{c,d} S_cd(q) d_d Vbar_c(q)
template <int D>
__global__ void __launch_bounds__(ZT) k_energy_rhs(ZoneArgs za, const double *__restrict__ Vb,
                                                   const double *__restrict__ Sq, const double *__restrict__ m1inv,
                                                   const double *__restrict__ zscale,
                                                   const double *__restrict__ Minv_dense, double *__restrict__ de) {
  extern __shared__ double sm[];
  const int k = za.k, n = 2 * k, p = k + 1, t = k;
  const int nk = ipow(p, D), nq = ipow(n, D), nt = ipow(t, D);
  double *B = sm, *G = B + n * p, *Phi = G + n * p, *Mi = Phi + n * t, *u = Mi + t * t, *Pq = u + D * nk;
  const int szT = D == 3 ? p * p * n : p * n, szX = D == 3 ? p * n * n : 0;
  double *TB = Pq + nq, *TG = TB + szT, *X0 = TG + szT, *X1 = X0 + szX, *X2 = X1 + szX;
  for (int i = threadIdx.x; i < 2 * n * p + n * t; i += blockDim.x) B[i] = za.tab[i];
  for (int i = threadIdx.x; i < t * t; i += blockDim.x) Mi[i] = m1inv[i];
  const int64_t z = blockIdx.x;
  const int32_t *zn = za.zone_nodes + z * nk;
  for (int i = threadIdx.x; i < D * nk; i += blockDim.x) {
    const int c = i / nk, a = i - c * nk;
    u[i] = Vb[(int64_t)c * za.nn + zn[a]];
  }
  for (int q = threadIdx.x; q < nq; q += blockDim.x) Pq[q] = 0.0;
  __syncthreads();
  const double *S = Sq + z * nq * D * D;
  for (int c = 0; c < D; ++c) {
    const double *uc = u + c * nk;
    if (D == 2) {
      contract<0>(uc, TB, p, p, 1, n, B, p, 1);
      contract<0>(uc, TG, p, p, 1, n, G, p, 1);
      __syncthreads();
      for (int q = threadIdx.x; q < nq; q += blockDim.x) {   // q = q0 + n q1
        const int q0 = q % n, q1 = q / n;
        double d0 = 0.0, d1 = 0.0;
        for (int i = 0; i < p; ++i) {
          d0 = fma(B[q1 * p + i], TG[i * n + q0], d0);
          d1 = fma(G[q1 * p + i], TB[i * n + q0], d1);
        }
        Pq[q] += S[(q * D + c) * D + 0] * d0 + S[(q * D + c) * D + 1] * d1;
      }
      __syncthreads();
    } else {
      contract<0>(uc, TB, p, p, p, n, B, p, 1);
      contract<0>(uc, TG, p, p, p, n, G, p, 1);
      __syncthreads();
      contract<1>(TG, X0, n, p, p, n, B, p, 1);   // d/dxi0
      contract<1>(TB, X1, n, p, p, n, G, p, 1);   // d/dxi1
      contract<1>(TB, X2, n, p, p, n, B, p, 1);   // d/dxi2 (after the last axis)
      __syncthreads();
      for (int q = threadIdx.x; q < nq; q += blockDim.x) {   // q = q0 + n (q1 + n q2)
        const int q01 = q % (n * n), q2 = q / (n * n);
        double d0 = 0.0, d1 = 0.0, d2 = 0.0;
        for (int i = 0; i < p; ++i) {
          const int src = i * n * n + q01;
          d0 = fma(B[q2 * p + i], X0[src], d0);
          d1 = fma(B[q2 * p + i], X1[src], d1);
          d2 = fma(G[q2 * p + i], X2[src], d2);
        }
        const double *s = S + (q * D + c) * D;
        Pq[q] += s[0] * d0 + s[1] * d1 + s[2] * d2;
      }
      __syncthreads();
    }
  }
  // project on phi_j: points -> [t]^D
  double *ftv = from_points<D>(Pq, D == 3 ? X0 : TB, Phi, n, t);
  // M_E^{-1}
  if (Minv_dense) {
    const double *Mz = Minv_dense + z * nt * nt;
    for (int i = threadIdx.x; i < nt; i += blockDim.x) {
      double s = 0.0;
      for (int j = 0; j < nt; ++j) s = fma(Mz[i * nt + j], ftv[j], s);
      de[z * nt + i] = s;
    }
  } else {
    double *a = ftv, *b = (ftv == TG) ? TB : TG;
    // forward with the [t][t] inverse: out(o) = sum_i Mi[o][i] in(i)
    if (D == 2) {
      contract<0>(a, b, t, t, 1, t, Mi, t, 1); __syncthreads();
      contract<1>(b, a, t, t, 1, t, Mi, t, 1); __syncthreads();
    } else {
      contract<0>(a, b, t, t, t, t, Mi, t, 1); __syncthreads();
      contract<1>(b, a, t, t, t, t, Mi, t, 1); __syncthreads();
      contract<2>(a, b, t, t, t, t, Mi, t, 1); __syncthreads();
      a = b;
    }
    const double sz = zscale[z];
    for (int i = threadIdx.x; i < nt; i += blockDim.x) de[z * nt + i] = a[i] * sz;
  }
}

// ------------------------------------------------------------------------------------------------
// per-node kernels
// ------------------------------------------------------------------------------------------------
struct NodeArgs {
  const int32_t *ptr, *ent;
  int64_t nn;
  int nk;
};

template <int D>
__device__ __forceinline__ void gather_node(const NodeArgs &na, const double *__restrict__ Y, int64_t node,
                                            double (&s)[D]) {
  const int b = na.ptr[node], e = na.ptr[node + 1];
#pragma unroll
  for (int c = 0; c < D; ++c) s[c] = 0.0;
  for (int i = b; i < e; ++i) {   // ascending zone id
    const int o = na.ent[i];
#pragma unroll
    for (int c = 0; c < D; ++c) s[c] += Y[o + c * na.nk];
  }
}

template <int D>
__global__ void __launch_bounds__(NB) k_gather(NodeArgs na, const double *__restrict__ Y, double *__restrict__ out) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= na.nn) return;
  double s[D];
  gather_node<D>(na, Y, n, s);
#pragma unroll
  for (int c = 0; c < D; ++c) out[c * na.nn + n] = s[c];
}

// CG start: X = 0, R = mask (sgn b), Z = R / diag, P = 0; rz, bb
template <int D, bool MULTI = false>
__global__ void __launch_bounds__(NB) k_cg_init(NodeArgs na, double sgn, const double *__restrict__ b,
                                                const double *__restrict__ invd, double *X, double *R, double *Zv,
                                                double *P, double *partials, CGScal *sc,
                                                const double *__restrict__ own = nullptr, double *red = nullptr) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  double v[2 * D];
#pragma unroll
  for (int c = 0; c < D; ++c) {
    double r = 0.0, zz = 0.0;
    if (n < na.nn) {
      const int64_t g = c * na.nn + n;
      const double id = invd[g];
      r = id != 0.0 ? sgn * b[g] : 0.0;
      zz = r * id;
      X[g] = 0.0; R[g] = r; Zv[g] = zz; P[g] = 0.0;
    }
    const double w = (MULTI && n < na.nn) ? own[n] : 1.0;   // each shared node counted by its owner only
    v[c] = w * r * zz;
    v[D + c] = w * r * r;
  }
  if (grid_sum<2 * D>(v, partials, &sc->ticket) && threadIdx.x == 0) {
    if (MULTI) {   // local sums; k_cg_scal finishes after the group allreduce
#pragma unroll
      for (int c = 0; c < 2 * D; ++c) red[c] = v[c];
      return;
    }
    bool done = true;
    for (int c = 0; c < D; ++c) {
      sc->rz[c] = v[c]; sc->bb[c] = v[D + c]; sc->rr[c] = v[D + c]; sc->beta[c] = 0.0; sc->alpha[c] = 0.0;
      done = done && v[D + c] == 0.0;
    }
    sc->done = done ? 1 : 0;
    sc->iters = 0;
  }
}

// AP = mask (sum of zone actions), P = Z + beta P; alpha = rz / (P . AP)
template <int D, bool DOT = true>
__global__ void __launch_bounds__(NB) k_cg_gather(NodeArgs na, const double *__restrict__ Y,
                                                  const double *__restrict__ invd, const double *__restrict__ Zv,
                                                  double *P, double *AP, double *partials, CGScal *sc) {
  if (sc->done) return;
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  double v[D];
#pragma unroll
  for (int c = 0; c < D; ++c) v[c] = 0.0;
  if (n < na.nn) {
    double s[D];
    gather_node<D>(na, Y, n, s);
#pragma unroll
    for (int c = 0; c < D; ++c) {
      const int64_t g = c * na.nn + n;
      const double pn = __fma_rn(sc->beta[c], P[g], Zv[g]);
      const double ap = invd[g] != 0.0 ? s[c] : 0.0;
      P[g] = pn;
      AP[g] = ap;
      v[c] = pn * ap;
    }
  }
  if (!DOT) return;   // multi-rank: AP still needs its shared-node sum before P . AP (k_cg_pap)
  if (grid_sum<D>(v, partials, &sc->ticket) && threadIdx.x == 0)
    for (int c = 0; c < D; ++c) sc->alpha[c] = v[c] > 0.0 ? sc->rz[c] / v[c] : 0.0;
}

// multi-rank: owned P . AP (after the shared-node sum of AP) -> red[0, D)
template <int D>
__global__ void __launch_bounds__(NB) k_cg_pap(int64_t nn, const double *__restrict__ P, const double *__restrict__ AP,
                                               const double *__restrict__ own, double *partials, CGScal *sc,
                                               double *red) {
  if (sc->done) return;
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  double v[D];
#pragma unroll
  for (int c = 0; c < D; ++c) v[c] = n < nn ? own[n] * P[c * nn + n] * AP[c * nn + n] : 0.0;
  if (grid_sum<D>(v, partials, &sc->ticket) && threadIdx.x == 0)
#pragma unroll
    for (int c = 0; c < D; ++c) red[c] = v[c];
}

// multi-rank scalar steps on the group-reduced sums (one thread):
//   PH 0 (after init): rz, bb, rr from red[0, 2D);  PH 1: alpha from red[0, D);  PH 2: beta, rr, done
template <int D, int PH>
__global__ void k_cg_scal(const double *__restrict__ red, CGScal *sc) {
  if (PH != 0 && sc->done) return;
  if (PH == 0) {
    bool done = true;
    for (int c = 0; c < D; ++c) {
      sc->rz[c] = red[c]; sc->bb[c] = red[D + c]; sc->rr[c] = red[D + c]; sc->beta[c] = 0.0; sc->alpha[c] = 0.0;
      done = done && red[D + c] == 0.0;
    }
    sc->done = done ? 1 : 0;
    sc->iters = 0;
  } else if (PH == 1) {
    for (int c = 0; c < D; ++c) sc->alpha[c] = red[c] > 0.0 ? sc->rz[c] / red[c] : 0.0;
  } else {
    bool done = true;
    for (int c = 0; c < D; ++c) {
      sc->beta[c] = sc->rz[c] > 0.0 ? red[c] / sc->rz[c] : 0.0;
      sc->rz[c] = red[c];
      sc->rr[c] = red[D + c];
      done = done && red[D + c] <= sc->tol2 * sc->bb[c];
    }
    sc->iters += 1;
    sc->done = done ? 1 : 0;
  }
}

// X += alpha P, R -= alpha AP, Z = R / diag; beta = rz' / rz; convergence
template <int D, bool MULTI = false>
__global__ void __launch_bounds__(NB) k_cg_update(NodeArgs na, const double *__restrict__ invd, double *X, double *R,
                                                  double *Zv, const double *__restrict__ P,
                                                  const double *__restrict__ AP, double *partials, CGScal *sc,
                                                  const double *__restrict__ own = nullptr, double *red = nullptr) {
  if (sc->done) return;
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  double v[2 * D];
#pragma unroll
  for (int c = 0; c < D; ++c) {
    double r = 0.0, zz = 0.0;
    if (n < na.nn) {
      const int64_t g = c * na.nn + n;
      const double al = sc->alpha[c];
      X[g] = fma(al, P[g], X[g]);
      r = fma(-al, AP[g], R[g]);
      zz = r * invd[g];
      R[g] = r; Zv[g] = zz;
    }
    const double w = (MULTI && n < na.nn) ? own[n] : 1.0;
    v[c] = w * r * zz;
    v[D + c] = w * r * r;
  }
  if (grid_sum<2 * D>(v, partials, &sc->ticket) && threadIdx.x == 0) {
    if (MULTI) {
#pragma unroll
      for (int c = 0; c < 2 * D; ++c) red[c] = v[c];
      return;
    }
    bool done = true;
    for (int c = 0; c < D; ++c) {
      sc->beta[c] = sc->rz[c] > 0.0 ? v[c] / sc->rz[c] : 0.0;
      sc->rz[c] = v[c];
      sc->rr[c] = v[D + c];
      done = done && v[D + c] <= sc->tol2 * sc->bb[c];
    }
    sc->iters += 1;
    sc->done = done ? 1 : 0;
  }
}

// out = a + h b (elementwise; out may alias a)
__global__ void __launch_bounds__(NB) k_axpy(double *out, const double *a, double h, const double *__restrict__ b,
                                             int64_t len) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < len; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = fma(h, b[i], a[i]);
}

// kinetic part: sum_c u_c . (gathered M u)_c  (halved on the host)
template <int D>
__global__ void __launch_bounds__(NB) k_gather_dot(NodeArgs na, const double *__restrict__ Y,
                                                   const double *__restrict__ u, double *partials, unsigned *ticket,
                                                   double *out, const double *__restrict__ own = nullptr) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  double v[1] = {0.0};
  if (n < na.nn) {
    double s[D];
    gather_node<D>(na, Y, n, s);
#pragma unroll
    for (int c = 0; c < D; ++c) v[0] += u[c * na.nn + n] * s[c];
    if (own) v[0] *= own[n];
  }
  if (grid_sum<1>(v, partials, ticket) && threadIdx.x == 0) *out = v[0];
}

// owner-weighted sum_c a_c . b_c over the local nodes ([dim][nn] vectors) -> *out
template <int D>
__global__ void __launch_bounds__(NB) k_wdot(int64_t nn, const double *__restrict__ a, const double *__restrict__ b,
                                             const double *__restrict__ own, double *partials, unsigned *ticket,
                                             double *out) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  double v[1] = {0.0};
  if (n < nn) {
#pragma unroll
    for (int c = 0; c < D; ++c) v[0] += a[c * nn + n] * b[c * nn + n];
    v[0] *= own[n];
  }
  if (grid_sum<1>(v, partials, ticket) && threadIdx.x == 0) *out = v[0];
}

__global__ void __launch_bounds__(NB) k_dot(const double *__restrict__ a, const double *__restrict__ b, int64_t len,
                                            double *partials, unsigned *ticket, double *out) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  double v[1] = {i < len ? a[i] * b[i] : 0.0};
  if (grid_sum<1>(v, partials, ticket) && threadIdx.x == 0) *out = v[0];
}

unsigned blocks_for(int64_t n, int t) { return (unsigned)std::max<int64_t>(1, (n + t - 1) / t); }

}  // namespace

// ------------------------------------------------------------------------------------------------
// handle
// ------------------------------------------------------------------------------------------------
struct blast_cf_rk2 {
  blast_cf *h = nullptr;
  HandleView hv{};
  blast_cf_rk2_opts opts{};
  int64_t nx = 0, ne = 0;
  // device
  double *R = nullptr, *Sq = nullptr, *F1 = nullptr, *FTv = nullptr, *dtd = nullptr;
  double *DV = nullptr, *Vb = nullptr, *DE = nullptr, *xh = nullptr, *eh = nullptr;
  double *bx = nullptr, *bv = nullptr, *be = nullptr;   // state backup for rejected steps (advance)
  double *Rr = nullptr, *Zv = nullptr, *P = nullptr, *AP = nullptr, *Y = nullptr, *invd = nullptr;
  double *partials = nullptr, *me1 = nullptr, *m1inv = nullptr, *zscale = nullptr, *Minv = nullptr;
  double *scal_out = nullptr;   // [4] energies / dots
  unsigned *ticket = nullptr;
  CGScal *sc = nullptr;
  // multi-rank: owner weights of the local nodes, group-reduction buffer
  bool multi = false, loopback = false, ready = false;
  double *own = nullptr, *red = nullptr;
  std::vector<unsigned char> fixed;   // [dim][nn] wall DOFs (host; the Jacobi diagonal is inverted after its shared-node sum)
  // host
  CGScal *h_sc = nullptr;   // pinned
  size_t smem_mass = 0, smem_diag = 0, smem_me1 = 0, smem_rhs = 0;
};

namespace {

void free_rk2(blast_cf_rk2 *s) {
  if (!s) return;
  double *bufs[] = {s->R, s->Sq, s->F1, s->FTv, s->dtd, s->DV, s->Vb, s->DE, s->xh, s->eh, s->Rr, s->Zv, s->P,
                    s->AP, s->Y, s->invd, s->partials, s->me1, s->m1inv, s->zscale, s->Minv, s->scal_out,
                    s->bx, s->bv, s->be, s->own, s->red};
  for (double *b : bufs) cudaFree(b);
  cudaFree(s->ticket);
  cudaFree(s->sc);
  if (s->h_sc) cudaFreeHost(s->h_sc);
  delete s;
}

ZoneArgs zone_args(const blast_cf_rk2 *s) {
  return ZoneArgs{s->hv.tab, s->hv.zone_nodes, s->R, s->hv.Z, s->hv.nn, s->hv.k};
}
NodeArgs node_args(const blast_cf_rk2 *s) { return NodeArgs{s->hv.ptr, s->hv.ent, s->hv.nn, s->hv.nk}; }

template <typename F>
int set_smem(F *f, size_t bytes) {
  if (bytes > 48 * 1024) CUDA_TRY(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes));
  return BLAST_CF_OK;
}

// M_V u per component into Y (zone-local)
void launch_mass_zone(blast_cf_rk2 *s, const double *u, const double *Pold, const CGScal *sc) {
  if (s->hv.Z == 0) return;
  if (s->hv.dim == 3)
    k_mass_zone<3><<<(unsigned)s->hv.Z, ZT, s->smem_mass, s->hv.stream>>>(zone_args(s), u, Pold, sc, s->Y);
  else
    k_mass_zone<2><<<(unsigned)s->hv.Z, ZT, s->smem_mass, s->hv.stream>>>(zone_args(s), u, Pold, sc, s->Y);
}

int check(const char *what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(BLAST_CF_ECUDA, "%s: %s", what, cudaGetErrorString(e));
  return BLAST_CF_OK;
}

int cg_solve(blast_cf_rk2 *s, const double *b, double sgn, double *X, int *iters_out);

// Multi-rank CG (f2): the group's ranks (n = 1 under NCCL, all n of a loopback group) run the same
// Jacobi PCG as cg_solve in lockstep; each iteration adds the shared-node sum of A p (the M_V action of a
// partition misses its neighbours' zones) and group sums of the owner-weighted dot products, so every
// rank holds the same scalars and, on shared nodes, bitwise the same iterates.
int cg_group(blast_cf_rk2 *const *S, int n, const double *const *b, double sgn, double *const *X, int *iters_out) {
  if (n == 1 && !S[0]->multi) return cg_solve(S[0], b[0], sgn, X[0], iters_out);
  std::vector<blast_cf *> hs(n);
  std::vector<double *> red(n), ap(n);
  for (int r = 0; r < n; ++r) { hs[r] = S[r]->h; red[r] = S[r]->red; ap[r] = S[r]->AP; }
  const int D = S[0]->hv.dim;
  int rc;
  for (int r = 0; r < n; ++r) {
    blast_cf_rk2 *s = S[r];
    const NodeArgs na = node_args(s);
    const unsigned nb = blocks_for(s->hv.nn, NB);
    if (D == 3) k_cg_init<3, true><<<nb, NB, 0, s->hv.stream>>>(na, sgn, b[r], s->invd, X[r], s->Rr, s->Zv, s->P, s->partials, s->sc, s->own, s->red);
    else k_cg_init<2, true><<<nb, NB, 0, s->hv.stream>>>(na, sgn, b[r], s->invd, X[r], s->Rr, s->Zv, s->P, s->partials, s->sc, s->own, s->red);
  }
  if ((rc = blastcf::group_allreduce(hs.data(), n, red.data(), 2 * D, 0))) return rc;
  for (int r = 0; r < n; ++r) {
    if (D == 3) k_cg_scal<3, 0><<<1, 1, 0, S[r]->hv.stream>>>(S[r]->red, S[r]->sc);
    else k_cg_scal<2, 0><<<1, 1, 0, S[r]->hv.stream>>>(S[r]->red, S[r]->sc);
  }
  int it = 0;
  const int every = std::max(1, S[0]->opts.cg_check_every);
  while (true) {
    CUDA_TRY(cudaMemcpyAsync(S[0]->h_sc, S[0]->sc, sizeof(CGScal), cudaMemcpyDeviceToHost, S[0]->hv.stream));
    CUDA_TRY(cudaStreamSynchronize(S[0]->hv.stream));
    if (S[0]->h_sc->done || it >= S[0]->opts.cg_max_iter) break;
    for (int j = 0; j < every && it < S[0]->opts.cg_max_iter; ++j, ++it) {
      for (int r = 0; r < n; ++r) {   // A p on every partition (p = z + beta p formed inside)
        blast_cf_rk2 *s = S[r];
        const unsigned nb = blocks_for(s->hv.nn, NB);
        launch_mass_zone(s, s->Zv, s->P, s->sc);
        if (D == 3) k_cg_gather<3, false><<<nb, NB, 0, s->hv.stream>>>(node_args(s), s->Y, s->invd, s->Zv, s->P, s->AP, s->partials, s->sc);
        else k_cg_gather<2, false><<<nb, NB, 0, s->hv.stream>>>(node_args(s), s->Y, s->invd, s->Zv, s->P, s->AP, s->partials, s->sc);
      }
      if ((rc = blastcf::group_exchange_sum(hs.data(), n, ap.data()))) return rc;
      for (int r = 0; r < n; ++r) {
        blast_cf_rk2 *s = S[r];
        const unsigned nb = blocks_for(s->hv.nn, NB);
        if (D == 3) k_cg_pap<3><<<nb, NB, 0, s->hv.stream>>>(s->hv.nn, s->P, s->AP, s->own, s->partials, s->sc, s->red);
        else k_cg_pap<2><<<nb, NB, 0, s->hv.stream>>>(s->hv.nn, s->P, s->AP, s->own, s->partials, s->sc, s->red);
      }
      if ((rc = blastcf::group_allreduce(hs.data(), n, red.data(), D, 0))) return rc;
      for (int r = 0; r < n; ++r) {
        blast_cf_rk2 *s = S[r];
        const unsigned nb = blocks_for(s->hv.nn, NB);
        if (D == 3) {
          k_cg_scal<3, 1><<<1, 1, 0, s->hv.stream>>>(s->red, s->sc);
          k_cg_update<3, true><<<nb, NB, 0, s->hv.stream>>>(node_args(s), s->invd, X[r], s->Rr, s->Zv, s->P, s->AP, s->partials, s->sc, s->own, s->red);
        } else {
          k_cg_scal<2, 1><<<1, 1, 0, s->hv.stream>>>(s->red, s->sc);
          k_cg_update<2, true><<<nb, NB, 0, s->hv.stream>>>(node_args(s), s->invd, X[r], s->Rr, s->Zv, s->P, s->AP, s->partials, s->sc, s->own, s->red);
        }
      }
      if ((rc = blastcf::group_allreduce(hs.data(), n, red.data(), 2 * D, 0))) return rc;
      for (int r = 0; r < n; ++r) {
        if (D == 3) k_cg_scal<3, 2><<<1, 1, 0, S[r]->hv.stream>>>(S[r]->red, S[r]->sc);
        else k_cg_scal<2, 2><<<1, 1, 0, S[r]->hv.stream>>>(S[r]->red, S[r]->sc);
      }
    }
    if ((rc = check("group CG kernels"))) return rc;
  }
  if (iters_out) *iters_out = S[0]->h_sc->iters;
  if (!S[0]->h_sc->done)
    return fail(BLAST_CF_EUNSUPPORTED, "CG did not converge in %d iterations (rel tol %g)", S[0]->opts.cg_max_iter,
                S[0]->opts.cg_rel_tol);
  return BLAST_CF_OK;
}

// X = M_V^{-1} (sgn b) on the free DOFs (fixed DOFs 0); returns iterations (max over components)
int cg_solve(blast_cf_rk2 *s, const double *b, double sgn, double *X, int *iters_out) {
  const HandleView &hv = s->hv;
  const NodeArgs na = node_args(s);
  const unsigned nb = blocks_for(hv.nn, NB);
  cudaStream_t st = hv.stream;
  if (hv.dim == 3)
    k_cg_init<3><<<nb, NB, 0, st>>>(na, sgn, b, s->invd, X, s->Rr, s->Zv, s->P, s->partials, s->sc);
  else
    k_cg_init<2><<<nb, NB, 0, st>>>(na, sgn, b, s->invd, X, s->Rr, s->Zv, s->P, s->partials, s->sc);
  int it = 0;
  const int every = std::max(1, s->opts.cg_check_every);
  while (true) {
    CUDA_TRY(cudaMemcpyAsync(s->h_sc, s->sc, sizeof(CGScal), cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaStreamSynchronize(st));
    if (s->h_sc->done || it >= s->opts.cg_max_iter) break;
    for (int j = 0; j < every && it < s->opts.cg_max_iter; ++j, ++it) {
      launch_mass_zone(s, s->Zv, s->P, s->sc);
      if (hv.dim == 3) {
        k_cg_gather<3><<<nb, NB, 0, st>>>(na, s->Y, s->invd, s->Zv, s->P, s->AP, s->partials, s->sc);
        k_cg_update<3><<<nb, NB, 0, st>>>(na, s->invd, X, s->Rr, s->Zv, s->P, s->AP, s->partials, s->sc);
      } else {
        k_cg_gather<2><<<nb, NB, 0, st>>>(na, s->Y, s->invd, s->Zv, s->P, s->AP, s->partials, s->sc);
        k_cg_update<2><<<nb, NB, 0, st>>>(na, s->invd, X, s->Rr, s->Zv, s->P, s->AP, s->partials, s->sc);
      }
    }
    int rc = check("CG kernels");
    if (rc) return rc;
  }
  if (iters_out) *iters_out = s->h_sc->iters;
  if (!s->h_sc->done)
    return fail(BLAST_CF_EUNSUPPORTED, "CG did not converge in %d iterations (rel tol %g)", s->opts.cg_max_iter,
                s->opts.cg_rel_tol);
  return BLAST_CF_OK;
}

void launch_energy_rhs(blast_cf_rk2 *s, const double *Vb, double *de) {
  if (s->hv.Z == 0) return;
  if (s->hv.dim == 3)
    k_energy_rhs<3><<<(unsigned)s->hv.Z, ZT, s->smem_rhs, s->hv.stream>>>(zone_args(s), Vb, s->Sq, s->m1inv,
                                                                          s->zscale, s->Minv, de);
  else
    k_energy_rhs<2><<<(unsigned)s->hv.Z, ZT, s->smem_rhs, s->hv.stream>>>(zone_args(s), Vb, s->Sq, s->m1inv,
                                                                          s->zscale, s->Minv, de);
}

void axpy(blast_cf_rk2 *s, double *out, const double *a, double h, const double *b, int64_t len) {
  if (len <= 0) return;
  k_axpy<<<(unsigned)std::min<int64_t>(blocks_for(len, NB), 148 * 16), NB, 0, s->hv.stream>>>(out, a, h, b, len);
}

// Gauss-Jordan inverse with partial pivoting, long double, in place on a[m][m]
bool invert_ld(std::vector<long double> &a, int m) {
  std::vector<long double> inv((size_t)m * m, 0.0L);
  for (int i = 0; i < m; ++i) inv[(size_t)i * m + i] = 1.0L;
  for (int col = 0; col < m; ++col) {
    int piv = col;
    for (int r = col + 1; r < m; ++r)
      if (fabsl(a[(size_t)r * m + col]) > fabsl(a[(size_t)piv * m + col])) piv = r;
    if (a[(size_t)piv * m + col] == 0.0L) return false;
    if (piv != col)
      for (int j = 0; j < m; ++j) {
        std::swap(a[(size_t)piv * m + j], a[(size_t)col * m + j]);
        std::swap(inv[(size_t)piv * m + j], inv[(size_t)col * m + j]);
      }
    const long double d = a[(size_t)col * m + col];
    for (int j = 0; j < m; ++j) { a[(size_t)col * m + j] /= d; inv[(size_t)col * m + j] /= d; }
    for (int r = 0; r < m; ++r) {
      if (r == col) continue;
      const long double f = a[(size_t)r * m + col];
      if (f == 0.0L) continue;
      for (int j = 0; j < m; ++j) {
        a[(size_t)r * m + j] -= f * a[(size_t)col * m + j];
        inv[(size_t)r * m + j] -= f * inv[(size_t)col * m + j];
      }
    }
  }
  a.swap(inv);
  return true;
}

// shared-node sum of the gathered mass diagonal over the group, then invd = 1/diag (0 on wall DOFs)
int finish_setup(blast_cf_rk2 *const *S, int n) {
  int rc;
  if (S[0]->multi) {
    std::vector<blast_cf *> hs(n);
    std::vector<double *> v(n);
    for (int r = 0; r < n; ++r) { hs[r] = S[r]->h; v[r] = S[r]->invd; }
    if ((rc = blastcf::group_exchange_sum(hs.data(), n, v.data()))) return rc;
  }
  for (int r = 0; r < n; ++r) {
    blast_cf_rk2 *s = S[r];
    const int64_t nx = s->nx;
    std::vector<double> diag(std::max<int64_t>(nx, 1), 0.0);
    if (nx > 0) CUDA_TRY(cudaMemcpyAsync(diag.data(), s->invd, nx * sizeof(double), cudaMemcpyDeviceToHost, s->hv.stream));
    CUDA_TRY(cudaStreamSynchronize(s->hv.stream));
    for (int64_t i = 0; i < nx; ++i) {
      double &d = diag[i];
      if (!(d > 0.0) && !s->fixed[i])
        return fail(BLAST_CF_EINVAL, "non-positive mass diagonal at DOF %lld of rank %d", (long long)i, r);
      d = s->fixed[i] ? 0.0 : 1.0 / d;
    }
    if (nx > 0) {   // ordered on the stream the CG kernels use (pageable source: wait for it)
      CUDA_TRY(cudaMemcpyAsync(s->invd, diag.data(), nx * sizeof(double), cudaMemcpyHostToDevice, s->hv.stream));
      CUDA_TRY(cudaStreamSynchronize(s->hv.stream));
    }
    s->ready = true;
  }
  return BLAST_CF_OK;
}

// dv/dt = -M_V^{-1} F.1 and de/dt = M_E^{-1} F^T vbar on every rank of the group
int rates_group(blast_cf_rk2 *const *S, int n, const double *const *x, const double *const *v, const double *const *e,
                const double *const *vbar, double *const *out_dvdt, double *const *out_dedt, double *out_dt,
                int32_t *cg_iters) {
  int rc;
  std::vector<blast_cf *> hs(n);
  std::vector<double *> f1(n), dtd(n);
  for (int r = 0; r < n; ++r) {
    blast_cf_rk2 *s = S[r];
    hs[r] = s->h; f1[r] = s->F1; dtd[r] = s->dtd;
    if ((rc = blastcf::eval_with_S(s->h, x[r], v[r], e[r], s->R, s->F1, s->FTv, s->dtd, s->Sq))) return rc;
  }
  if (S[0]->loopback) {   // (an NCCL rank's evaluation already summed F.1 and reduced dt)
    if ((rc = blastcf::group_exchange_sum(hs.data(), n, f1.data()))) return rc;
    if ((rc = blastcf::group_allreduce(hs.data(), n, dtd.data(), 1, 1))) return rc;
  }
  int it = 0;
  if ((rc = cg_group(S, n, f1.data(), -1.0, out_dvdt, &it))) return rc;
  if (cg_iters) *cg_iters = it;
  for (int r = 0; r < n; ++r) launch_energy_rhs(S[r], vbar && vbar[r] ? vbar[r] : v[r], out_dedt[r]);
  if ((rc = check("energy rhs"))) return rc;
  if (out_dt) CUDA_TRY(cudaMemcpyAsync(out_dt, S[0]->dtd, sizeof(double), cudaMemcpyDeviceToHost, S[0]->hv.stream));
  for (int r = 0; r < n; ++r) CUDA_TRY(cudaStreamSynchronize(S[r]->hv.stream));
  return BLAST_CF_OK;
}

// kinetic = 1/2 sum_c v_c^T M_V v_c and internal = sum_z 1^T M_E e_z over the whole group (shared nodes:
// (M_V v) summed over their sharers, then counted by the owner)
int energy_group(blast_cf_rk2 *const *S, int n, const double *const *v, const double *const *e, double *kinetic,
                 double *internal) {
  int rc;
  std::vector<blast_cf *> hs(n);
  std::vector<double *> ap(n), out(n);
  for (int r = 0; r < n; ++r) {
    blast_cf_rk2 *s = S[r];
    hs[r] = s->h; ap[r] = s->AP; out[r] = s->scal_out;
    cudaStream_t st = s->hv.stream;
    CUDA_TRY(cudaMemsetAsync(s->scal_out, 0, 2 * sizeof(double), st));
    launch_mass_zone(s, v[r], nullptr, nullptr);
    if (s->hv.nn > 0) {
      if (s->multi) {   // M_V v to the nodes; its dot with v after the shared-node sum
        if (s->hv.dim == 3) k_gather<3><<<blocks_for(s->hv.nn, NB), NB, 0, st>>>(node_args(s), s->Y, s->AP);
        else k_gather<2><<<blocks_for(s->hv.nn, NB), NB, 0, st>>>(node_args(s), s->Y, s->AP);
      } else if (s->hv.dim == 3) {
        k_gather_dot<3><<<blocks_for(s->hv.nn, NB), NB, 0, st>>>(node_args(s), s->Y, v[r], s->partials, s->ticket, s->scal_out);
      } else {
        k_gather_dot<2><<<blocks_for(s->hv.nn, NB), NB, 0, st>>>(node_args(s), s->Y, v[r], s->partials, s->ticket, s->scal_out);
      }
    }
    if (s->ne > 0) k_dot<<<blocks_for(s->ne, NB), NB, 0, st>>>(s->me1, e[r], s->ne, s->partials, s->ticket, s->scal_out + 1);
  }
  if (S[0]->multi) {
    if ((rc = blastcf::group_exchange_sum(hs.data(), n, ap.data()))) return rc;
    for (int r = 0; r < n; ++r) {
      blast_cf_rk2 *s = S[r];
      if (s->hv.nn == 0) continue;
      if (s->hv.dim == 3) k_wdot<3><<<blocks_for(s->hv.nn, NB), NB, 0, s->hv.stream>>>(s->hv.nn, v[r], s->AP, s->own, s->partials, s->ticket, s->scal_out);
      else k_wdot<2><<<blocks_for(s->hv.nn, NB), NB, 0, s->hv.stream>>>(s->hv.nn, v[r], s->AP, s->own, s->partials, s->ticket, s->scal_out);
    }
    if ((rc = blastcf::group_allreduce(hs.data(), n, out.data(), 2, 0))) return rc;
  }
  if ((rc = check("energy"))) return rc;
  double res[2];
  CUDA_TRY(cudaMemcpyAsync(res, S[0]->scal_out, sizeof res, cudaMemcpyDeviceToHost, S[0]->hv.stream));
  for (int r = 0; r < n; ++r) CUDA_TRY(cudaStreamSynchronize(S[r]->hv.stream));
  *kinetic = 0.5 * res[0];
  *internal = res[1];
  return BLAST_CF_OK;
}

}  // namespace

extern "C" {

void blast_cf_rk2_default_opts(blast_cf_rk2_opts *o) {
  if (!o) return;
  o->cg_rel_tol = 1e-14;
  o->cg_max_iter = 500;
  o->cg_check_every = 8;
  o->wall_bc = 1;
  for (int c = 0; c < 3; ++c) o->box_lo[c] = o->box_hi[c] = 0.0;   // not given: derived at create
}

int blast_cf_rk2_create(blast_cf *h, const blast_cf_mesh *mesh, const double *rho0detJ0,
                        const blast_cf_rk2_opts *opts, blast_cf_rk2 **out) {
  if (!out) return fail(BLAST_CF_EINVAL, "out is NULL");
  *out = nullptr;
  if (!h || !mesh) return fail(BLAST_CF_EINVAL, "NULL argument");
  blast_cf_rk2 *s = new (std::nothrow) blast_cf_rk2();
  if (!s) return fail(BLAST_CF_ENOMEM, "host allocation");
  auto bail = [&](int code) { free_rk2(s); return code; };
  int rc = blastcf::handle_view(h, &s->hv);
  if (rc) return bail(rc);
  const HandleView &hv = s->hv;
  s->multi = hv.multi_rank;
  s->loopback = hv.loopback;
  if (mesh->num_zones != hv.Z || mesh->num_nodes != hv.nn || mesh->dim != hv.dim || mesh->order != hv.k)
    return bail(fail(BLAST_CF_EINVAL, "mesh does not match the handle"));
  if (hv.Z > 0 && !rho0detJ0) return bail(fail(BLAST_CF_EINVAL, "rho0detJ0 is NULL"));
  s->h = h;
  if (opts) s->opts = *opts; else blast_cf_rk2_default_opts(&s->opts);
  if (!(s->opts.cg_rel_tol > 0.0) || s->opts.cg_max_iter < 1) return bail(fail(BLAST_CF_EINVAL, "cg options"));
  const int D = hv.dim, k = hv.k, n = 2 * k, p = k + 1, t = k;
  const int64_t Z = hv.Z, nn = hv.nn;
  s->nx = (int64_t)D * nn;
  s->ne = Z * hv.nt;
  const size_t nx = std::max<int64_t>(s->nx, 1), ne = std::max<int64_t>(s->ne, 1);
  const size_t nzq = std::max<int64_t>(Z * hv.nq, 1), nzk = std::max<int64_t>(Z * D * hv.nk, 1);
  const unsigned nb = blocks_for(std::max<int64_t>(nn, s->ne), NB);

  // shared-memory footprints (doubles) of the zone kernels
  const size_t nq = hv.nq, nk = hv.nk;
  s->smem_mass = (n * p + n + 3 * nq) * sizeof(double);
  s->smem_diag = (n * p + n + 2 * nq) * sizeof(double);
  s->smem_me1 = (n * t + n + 2 * nq) * sizeof(double);
  const size_t szT = D == 3 ? (size_t)p * p * n : (size_t)p * n, szX = D == 3 ? (size_t)p * n * n : 0;
  s->smem_rhs = (2 * n * p + n * t + t * t + D * nk + nq + 2 * szT + 3 * szX) * sizeof(double);
  if (D == 3) {
    if ((rc = set_smem(k_mass_zone<3>, s->smem_mass)) || (rc = set_smem(k_diag_zone<3>, s->smem_diag)) ||
        (rc = set_smem(k_me1_zone<3>, s->smem_me1)) || (rc = set_smem(k_energy_rhs<3>, s->smem_rhs)))
      return bail(rc);
  } else {
    if ((rc = set_smem(k_mass_zone<2>, s->smem_mass)) || (rc = set_smem(k_diag_zone<2>, s->smem_diag)) ||
        (rc = set_smem(k_me1_zone<2>, s->smem_me1)) || (rc = set_smem(k_energy_rhs<2>, s->smem_rhs)))
      return bail(rc);
  }

  // ---- allocations ----
  double **dbl[] = {&s->F1, &s->DV, &s->Vb, &s->xh, &s->Rr, &s->Zv, &s->P, &s->AP, &s->invd, &s->bx, &s->bv};
  for (double **b : dbl) CUDA_TRY(cudaMalloc(b, nx * sizeof(double)));
  double **ebl[] = {&s->FTv, &s->DE, &s->eh, &s->me1, &s->be};
  for (double **b : ebl) CUDA_TRY(cudaMalloc(b, ne * sizeof(double)));
  CUDA_TRY(cudaMalloc(&s->R, nzq * sizeof(double)));
  CUDA_TRY(cudaMalloc(&s->Sq, nzq * D * D * sizeof(double)));
  CUDA_TRY(cudaMalloc(&s->Y, nzk * sizeof(double)));
  CUDA_TRY(cudaMalloc(&s->dtd, 2 * sizeof(double)));
  CUDA_TRY(cudaMalloc(&s->partials, (size_t)nb * 2 * D * sizeof(double)));
  CUDA_TRY(cudaMalloc(&s->scal_out, 4 * sizeof(double)));
  CUDA_TRY(cudaMalloc(&s->ticket, sizeof(unsigned)));
  CUDA_TRY(cudaMemset(s->ticket, 0, sizeof(unsigned)));
  CUDA_TRY(cudaMalloc(&s->sc, sizeof(CGScal)));
  CUDA_TRY(cudaMemset(s->sc, 0, sizeof(CGScal)));
  CUDA_TRY(cudaMallocHost(&s->h_sc, sizeof(CGScal)));
  CUDA_TRY(cudaMalloc(&s->red, (2 * D + 2) * sizeof(double)));
  if (s->multi) {
    std::vector<double> own(std::max<int64_t>(nn, 1), 1.0);
    if ((rc = blastcf::owner_weights(h, own.data()))) return bail(rc);
    CUDA_TRY(cudaMalloc(&s->own, own.size() * sizeof(double)));
    CUDA_TRY(cudaMemcpy(s->own, own.data(), own.size() * sizeof(double), cudaMemcpyHostToDevice));
  }
  CUDA_TRY(cudaMalloc(&s->m1inv, (size_t)t * t * sizeof(double)));
  CUDA_TRY(cudaMalloc(&s->zscale, std::max<int64_t>(Z, 1) * sizeof(double)));
  if (Z > 0) CUDA_TRY(cudaMemcpy(s->R, rho0detJ0, (size_t)Z * hv.nq * sizeof(double), cudaMemcpyHostToDevice));
  {
    const double tol2 = s->opts.cg_rel_tol * s->opts.cg_rel_tol;
    CUDA_TRY(cudaMemcpy(&s->sc->tol2, &tol2, sizeof tol2, cudaMemcpyHostToDevice));
  }

  // ---- M_E^{-1}: 1-D inverse (tensor zones) or dense per-zone inverses ----
  const blastcf::Tables1D T = blastcf::build_tables(k);
  {
    std::vector<long double> M1((size_t)t * t, 0.0L);
    for (int i = 0; i < t; ++i)
      for (int j = 0; j < t; ++j)
        for (int q = 0; q < n; ++q)
          M1[(size_t)i * t + j] += (long double)T.qwt[q] * T.Phi[q * t + i] * T.Phi[q * t + j];
    if (!invert_ld(M1, t)) return bail(fail(BLAST_CF_EINVAL, "1-D thermodynamic mass matrix is singular"));
    std::vector<double> m1d(M1.begin(), M1.end());
    CUDA_TRY(cudaMemcpy(s->m1inv, m1d.data(), m1d.size() * sizeof(double), cudaMemcpyHostToDevice));
  }
  std::vector<double> zscale(std::max<int64_t>(Z, 1), 0.0);
  bool all_uniform = true;
  for (int64_t z = 0; z < Z && all_uniform; ++z) {
    const double *r = rho0detJ0 + z * hv.nq;
    for (int q = 1; q < hv.nq; ++q)
      if (fabs(r[q] - r[0]) > 4e-16 * fabs(r[0])) { all_uniform = false; break; }
    if (!(r[0] > 0.0)) return bail(fail(BLAST_CF_EINVAL, "rho0detJ0 of zone %lld is not positive", (long long)z));
    zscale[z] = 1.0 / r[0];
  }
  if (all_uniform) {
    CUDA_TRY(cudaMemcpy(s->zscale, zscale.data(), zscale.size() * sizeof(double), cudaMemcpyHostToDevice));
  } else {
    const int nt = hv.nt, nqq = hv.nq;
    const double cost = (double)Z * ((double)nt * nt * nt + (double)nqq * nt * nt);
    if (cost > 17179869184.0)
      return bail(fail(BLAST_CF_EUNSUPPORTED, "dense M_E^{-1} for %lld zones of Nt=%d exceeds the create budget",
                       (long long)Z, nt));
    // dense phi and alpha at the points
    std::vector<double> phi((size_t)nqq * nt), al(nqq);
    for (int q = 0; q < nqq; ++q) {
      const int qi[3] = {q % n, (q / n) % n, q / (n * n)};
      double a = 1.0;
      for (int d = 0; d < D; ++d) a *= T.qwt[qi[d]];
      al[q] = a;
      for (int j = 0; j < nt; ++j) {
        const int ji[3] = {j % t, (j / t) % t, j / (t * t)};
        double f = 1.0;
        for (int d = 0; d < D; ++d) f *= T.Phi[qi[d] * t + ji[d]];
        phi[(size_t)q * nt + j] = f;
      }
    }
    std::vector<double> Minv((size_t)Z * nt * nt);
    std::vector<long double> M((size_t)nt * nt);
    for (int64_t z = 0; z < Z; ++z) {
      std::fill(M.begin(), M.end(), 0.0L);
      for (int q = 0; q < nqq; ++q) {
        const long double w = (long double)al[q] * rho0detJ0[z * nqq + q];
        for (int i = 0; i < nt; ++i)
          for (int j = 0; j < nt; ++j) M[(size_t)i * nt + j] += w * phi[(size_t)q * nt + i] * phi[(size_t)q * nt + j];
      }
      if (!invert_ld(M, nt)) return bail(fail(BLAST_CF_EINVAL, "M_E of zone %lld is singular", (long long)z));
      for (size_t i = 0; i < M.size(); ++i) Minv[(size_t)z * nt * nt + i] = (double)M[i];
    }
    CUDA_TRY(cudaMalloc(&s->Minv, Minv.size() * sizeof(double)));
    CUDA_TRY(cudaMemcpy(s->Minv, Minv.data(), Minv.size() * sizeof(double), cudaMemcpyHostToDevice));
  }

  // ---- Jacobi diagonal, walls, internal-energy weights ----
  // the uploads above are legacy-stream copies from pageable memory: let them land before kernels on hv.stream
  CUDA_TRY(cudaDeviceSynchronize());
  cudaStream_t st = hv.stream;
  if (Z > 0) {
    if (D == 3) {
      k_diag_zone<3><<<(unsigned)Z, ZT, s->smem_diag, st>>>(zone_args(s), s->Y);
      k_me1_zone<3><<<(unsigned)Z, ZT, s->smem_me1, st>>>(zone_args(s), s->me1);
    } else {
      k_diag_zone<2><<<(unsigned)Z, ZT, s->smem_diag, st>>>(zone_args(s), s->Y);
      k_me1_zone<2><<<(unsigned)Z, ZT, s->smem_me1, st>>>(zone_args(s), s->me1);
    }
  }
  if (nn > 0) {
    if (D == 3) k_gather<3><<<blocks_for(nn, NB), NB, 0, st>>>(node_args(s), s->Y, s->invd);
    else k_gather<2><<<blocks_for(nn, NB), NB, 0, st>>>(node_args(s), s->Y, s->invd);
  }
  if ((rc = check("create kernels"))) return bail(rc);
  // walls (reading R23): the faces of the GLOBAL box.  Given in opts, else the bounding box of x0 (one
  // rank) or its group min / max (NCCL ranks); a loopback group must pass it (no collective at create).
  double lo[3], hi[3];
  const bool given = s->opts.box_hi[0] > s->opts.box_lo[0];
  for (int c = 0; c < D; ++c) {
    lo[c] = given ? s->opts.box_lo[c] : HUGE_VAL;
    hi[c] = given ? s->opts.box_hi[c] : -HUGE_VAL;
    for (int64_t i = 0; i < nn && !given; ++i) { lo[c] = std::min(lo[c], mesh->x0[c * nn + i]); hi[c] = std::max(hi[c], mesh->x0[c * nn + i]); }
  }
  if (s->multi && !given && s->opts.wall_bc) {
    if (s->loopback) return bail(fail(BLAST_CF_EINVAL, "a loopback group needs opts->box_lo/box_hi (the global box)"));
    double mm[6] = {0, 0, 0, 0, 0, 0};
    for (int c = 0; c < D; ++c) { mm[c] = -lo[c]; mm[3 + c] = hi[c]; }
    CUDA_TRY(cudaMemcpyAsync(s->red, mm, 6 * sizeof(double), cudaMemcpyHostToDevice, st));
    CUDA_TRY(cudaStreamSynchronize(st));
    blast_cf *hh = h;
    double *rb = s->red;
    if ((rc = blastcf::group_allreduce(&hh, 1, &rb, 6, 2))) return bail(rc);
    CUDA_TRY(cudaStreamSynchronize(st));
    CUDA_TRY(cudaMemcpyAsync(mm, s->red, 6 * sizeof(double), cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaStreamSynchronize(st));
    for (int c = 0; c < D; ++c) { lo[c] = -mm[c]; hi[c] = mm[3 + c]; }
  }
  s->fixed.assign(nx, 0);
  for (int c = 0; c < D; ++c) {
    const double tol = 1e-12 * (hi[c] - lo[c]);
    for (int64_t i = 0; i < nn; ++i) {
      const double xv = mesh->x0[c * nn + i];
      s->fixed[c * nn + i] = s->opts.wall_bc && (fabs(xv - lo[c]) <= tol || fabs(xv - hi[c]) <= tol);
    }
  }
  // the Jacobi diagonal: shared-node sum first (a partition's zones give only part of a shared node's
  // diagonal), then inverted with the wall mask; a loopback group does that in blast_cf_rk2_setup_loopback
  if (!s->loopback) {
    blast_cf_rk2 *one = s;
    if ((rc = finish_setup(&one, 1))) return bail(rc);
  }
  *out = s;
  return BLAST_CF_OK;
}

int blast_cf_rk2_rates(blast_cf_rk2 *s, const double *x, const double *v, const double *e, const double *vbar,
                       double *out_dvdt, double *out_dedt, double *out_dt, int32_t *cg_iters) {
  if (!s || !out_dvdt || !out_dedt) return fail(BLAST_CF_EINVAL, "NULL argument");
  if (s->loopback) return fail(BLAST_CF_EINVAL, "loopback group: use blast_cf_rk2_rates_loopback");
  return rates_group(&s, 1, &x, &v, &e, &vbar, &out_dvdt, &out_dedt, out_dt, cg_iters);
}

int blast_cf_rk2_rates_loopback(blast_cf_rk2 *const *S, int n, const double *const *x, const double *const *v,
                                const double *const *e, const double *const *vbar, double *const *out_dvdt,
                                double *const *out_dedt, double *out_dt, int32_t *cg_iters) {
  if (!S || n < 1 || !x || !v || !e || !out_dvdt || !out_dedt) return fail(BLAST_CF_EINVAL, "NULL argument");
  for (int r = 0; r < n; ++r)
    if (!S[r] || !S[r]->loopback || S[r]->hv.rank != r || S[r]->hv.nranks != n || !S[r]->ready)
      return fail(BLAST_CF_EINVAL, "integrator %d is not rank %d of a set-up %d-rank loopback group", r, r, n);
  return rates_group(S, n, x, v, e, vbar, out_dvdt, out_dedt, out_dt, cg_iters);
}

int blast_cf_rk2_setup_loopback(blast_cf_rk2 *const *S, int n) {
  if (!S || n < 1) return fail(BLAST_CF_EINVAL, "NULL argument");
  for (int r = 0; r < n; ++r)
    if (!S[r] || !S[r]->loopback || S[r]->hv.rank != r || S[r]->hv.nranks != n)
      return fail(BLAST_CF_EINVAL, "integrator %d is not rank %d of a %d-rank loopback group", r, r, n);
  return finish_setup(S, n);
}

int blast_cf_rk2_energy_loopback(blast_cf_rk2 *const *S, int n, const double *const *v, const double *const *e,
                                 double *kinetic, double *internal) {
  if (!S || n < 1 || !v || !e || !kinetic || !internal) return fail(BLAST_CF_EINVAL, "NULL argument");
  for (int r = 0; r < n; ++r)
    if (!S[r] || !S[r]->loopback || S[r]->hv.rank != r || S[r]->hv.nranks != n)
      return fail(BLAST_CF_EINVAL, "integrator %d is not rank %d of a %d-rank loopback group", r, r, n);
  return energy_group(S, n, v, e, kinetic, internal);
}

int blast_cf_rk2_step(blast_cf_rk2 *s, double *x, double *v, double *e, double dt, double *dt_est,
                      int32_t *cg_iters) {
  if (!s || ((!x || !v) && s->nx > 0) || (!e && s->ne > 0)) return fail(BLAST_CF_EINVAL, "NULL argument");
  if (s->loopback) return fail(BLAST_CF_EINVAL, "loopback group: step the ranks with blast_cf_rk2_rates_loopback");
  const double h = 0.5 * dt;
  int rc, it0 = 0, it1 = 0;
  cudaStream_t st = s->hv.stream;
  // stage 1 at S0
  if ((rc = blastcf::eval_with_S(s->h, x, v, e, s->R, s->F1, s->FTv, s->dtd, s->Sq))) return rc;
  if ((rc = cg_group(&s, 1, &s->F1, -1.0, &s->DV, &it0))) return rc;
  axpy(s, s->Vb, v, h, s->DV, s->nx);                    // Vb = v0 + dt/2 dv0
  launch_energy_rhs(s, s->Vb, s->DE);                    // de0 = M_E^{-1} F(S0)^T Vb
  axpy(s, s->xh, x, h, s->Vb, s->nx);                    // x_half
  axpy(s, s->eh, e, h, s->DE, s->ne);                    // e_half
  // stage 2 at S_half = (x_half, Vb, e_half)
  if ((rc = blastcf::eval_with_S(s->h, s->xh, s->Vb, s->eh, s->R, s->F1, s->FTv, s->dtd + 1, s->Sq))) return rc;
  if ((rc = cg_group(&s, 1, &s->F1, -1.0, &s->DV, &it1))) return rc;
  axpy(s, s->Vb, v, h, s->DV, s->nx);                    // Vb = v0 + dt/2 dv1
  launch_energy_rhs(s, s->Vb, s->DE);                    // de1
  axpy(s, x, x, dt, s->Vb, s->nx);
  axpy(s, v, v, dt, s->DV, s->nx);
  axpy(s, e, e, dt, s->DE, s->ne);
  if ((rc = check("rk2 step"))) return rc;
  double dts[2] = {HUGE_VAL, HUGE_VAL};
  CUDA_TRY(cudaMemcpyAsync(dts, s->dtd, 2 * sizeof(double), cudaMemcpyDeviceToHost, st));
  CUDA_TRY(cudaStreamSynchronize(st));
  if (dt_est) *dt_est = std::min(dts[0], dts[1]);
  if (cg_iters) *cg_iters = it0 + it1;
  return BLAST_CF_OK;
}

int blast_cf_rk2_advance(blast_cf_rk2 *s, double *x, double *v, double *e, double t_final, int32_t max_steps,
                         double *dt, double *t_reached, int32_t *steps, int32_t *rejected) {
  if (!s || !dt || ((!x || !v) && s->nx > 0) || (!e && s->ne > 0)) return fail(BLAST_CF_EINVAL, "NULL argument");
  if (!(*dt > 0.0)) return fail(BLAST_CF_EINVAL, "dt must be positive");
  cudaStream_t st = s->hv.stream;
  const size_t bx = (size_t)s->nx * sizeof(double), be = (size_t)s->ne * sizeof(double);
  double t = 0.0, d = *dt;
  int32_t nst = 0, nrej = 0;
  int rc = BLAST_CF_OK;
  while (t < t_final && nst < max_steps) {
    const double dt_use = std::min(d, t_final - t);
    if (bx) { CUDA_TRY(cudaMemcpyAsync(s->bx, x, bx, cudaMemcpyDeviceToDevice, st));
              CUDA_TRY(cudaMemcpyAsync(s->bv, v, bx, cudaMemcpyDeviceToDevice, st)); }
    if (be) CUDA_TRY(cudaMemcpyAsync(s->be, e, be, cudaMemcpyDeviceToDevice, st));
    double dte = 0.0;
    if ((rc = blast_cf_rk2_step(s, x, v, e, dt_use, &dte, nullptr))) return rc;
    if (dte < dt_use) {   // reject: restore and retry with a smaller step
      if (bx) { CUDA_TRY(cudaMemcpyAsync(x, s->bx, bx, cudaMemcpyDeviceToDevice, st));
                CUDA_TRY(cudaMemcpyAsync(v, s->bv, bx, cudaMemcpyDeviceToDevice, st)); }
      if (be) CUDA_TRY(cudaMemcpyAsync(e, s->be, be, cudaMemcpyDeviceToDevice, st));
      d = 0.85 * dt_use;
      ++nrej;
      if (!(d > 1e-300)) return fail(BLAST_CF_EINVAL, "time step collapsed to zero");
      continue;
    }
    t += dt_use;
    ++nst;
    d = dte >= 1.25 * dt_use ? 1.02 * dt_use : dt_use;
  }
  CUDA_TRY(cudaStreamSynchronize(st));
  *dt = d;
  if (t_reached) *t_reached = t;
  if (steps) *steps = nst;
  if (rejected) *rejected = nrej;
  return BLAST_CF_OK;
}

int blast_cf_rk2_mass_apply(blast_cf_rk2 *s, const double *u, double *out) {
  if (!s || ((!u || !out) && s->nx > 0)) return fail(BLAST_CF_EINVAL, "NULL argument");
  launch_mass_zone(s, u, nullptr, nullptr);
  if (s->hv.nn > 0) {
    if (s->hv.dim == 3) k_gather<3><<<blocks_for(s->hv.nn, NB), NB, 0, s->hv.stream>>>(node_args(s), s->Y, out);
    else k_gather<2><<<blocks_for(s->hv.nn, NB), NB, 0, s->hv.stream>>>(node_args(s), s->Y, out);
  }
  int rc = check("mass apply");
  if (rc) return rc;
  CUDA_TRY(cudaStreamSynchronize(s->hv.stream));
  return BLAST_CF_OK;
}

int blast_cf_rk2_energy(blast_cf_rk2 *s, const double *v, const double *e, double *kinetic, double *internal) {
  if (!s || !kinetic || !internal) return fail(BLAST_CF_EINVAL, "NULL argument");
  if (s->loopback) return fail(BLAST_CF_EINVAL, "loopback group: use blast_cf_rk2_energy_loopback");
  return energy_group(&s, 1, &v, &e, kinetic, internal);
}

int blast_cf_rk2_destroy(blast_cf_rk2 *s) {
  if (!s) return fail(BLAST_CF_EINVAL, "NULL handle");
  cudaStreamSynchronize(s->hv.stream);
  free_rk2(s);
  return BLAST_CF_OK;
}

}  // extern "C"
