// KB1 v2 — 3D corner force for orders k <= 4 with whole-zone sum-factorization stages.
//
// Same mathematics as kb1_corner_force.cuh (eq (4)-(6); the a0..a5 rows of DESIGN.md §1), laid
// out for the FP64 pipe instead of the shared-memory pipe:
//   * every contraction stage runs over ALL quadrature slabs at once (7 barriers per zone instead of
//     5 per slab), so each work item loads its p (or n) inputs once into registers and produces
//     2n / 3n / p outputs from them (8-16 FMAs per shared-memory load);
//   * the 1-D tables are read from the constant bank with compile-time indices (the FMA takes them as
//     an immediate c[][] operand: no load instruction at all), except where the index is per-thread
//     (stage C, the point's own q0) where they come from a shared-memory copy;
//   * one thread owns two quadrature points (q0 and q0 + n/2 of the same (q1, q2) column) and runs the
//     point evaluation for each in turn, so a CTA of ZPC zones has ZPC * Nq / 2 threads.
//
// Shared memory per zone, two regions that are reused as the stages retire their inputs:
//   R0: X[6][P^3] E[T^3] T[6][2][N][P^2] TE[N][T^2]  ->  S,Pq of points q0 < N/2  ->  Z[3][2][N][P^2] ZE[N][T^2]
//   R1: U[6][3][N][N][P] UE[N][N][T]                 ->  S,Pq of points q0 >= N/2 + Y[9][P][N][N] YE[T][N][N]
#pragma once
#include "kb1_corner_force.cuh"

constexpr int ctab_size(int k) { return 2 * (2 * k) * (k + 1) + (2 * k) * k + 2 * k; }
constexpr int ctab_off(int k) { return k <= 1 ? 0 : ctab_off(k - 1) + ctab_size(k - 1); }
constexpr int CTAB_TOTAL = ctab_off(9);
__constant__ double c_tabs[CTAB_TOTAL];   // per order k: B[N][P] G[N][P] Phi[N][T] W[N] (tables.h)

template <int K>
struct CT {
  static constexpr int N = 2 * K, P = K + 1, T = K, OFF = ctab_off(K);
  static __device__ __forceinline__ double B(int q, int a) { return c_tabs[OFF + q * P + a]; }
  static __device__ __forceinline__ double G(int q, int a) { return c_tabs[OFF + N * P + q * P + a]; }
  static __device__ __forceinline__ double Phi(int q, int j) { return c_tabs[OFF + 2 * N * P + q * T + j]; }
  static __device__ __forceinline__ double W(int q) { return c_tabs[OFF + 2 * N * P + N * T + q]; }
};

template <int K>
struct V2Dims {
  static constexpr int N = 2 * K, P = K + 1, T = K;
  static constexpr int P2 = P * P, P3 = P * P * P, T2 = T * T, T3 = T * T * T, N2 = N * N, N3 = N * N * N;
  static constexpr int NQ = N3, TPZ = N3 / 2;
  static constexpr int NH = N / 2, SH = 10 * N2 * NH;   // S[9] + Pq for half of the points
  // PF (x2, double-buffered, filled by cp.async one batch ahead): X/V[6][P^3] E[T^3] R[N^3] J0^{-1}[9] gamma
  static constexpr int PF_X = 0, PF_E = 6 * P3, PF_R = PF_E + T3, PF_J = PF_R + N3;
  static constexpr int PFZ = (PF_J + 10 + 1) / 2 * 2;   // keep 16-byte alignment of every zone's block
  // R0: forward T, TE  ->  S/Pq of the points q0 < N/2  ->  Z, ZE
  static constexpr int O_T = 0, O_TE = O_T + 12 * N * P2;
  static constexpr int R0_FWD = O_TE + N * T2;
  static constexpr int O_SA = 0;
  static constexpr int O_Z = 0, O_ZE = 6 * N * P2;
  static constexpr int R0_Z = O_ZE + N * T2;
  static constexpr int R0 = R0_FWD > SH ? (R0_FWD > R0_Z ? R0_FWD : R0_Z) : (SH > R0_Z ? SH : R0_Z);
  // R1: forward U, UE  ->  S/Pq of the points q0 >= N/2, then Y, YE behind them
  static constexpr int O_U = 0, O_UE = 18 * N2 * P;
  static constexpr int R1_FWD = O_UE + N2 * T;
  static constexpr int O_SB = 0, O_Y = SH, O_YE = O_Y + 9 * P * N2;
  static constexpr int R1_BCK = O_YE + T * N2;
  static constexpr int R1 = R1_FWD > R1_BCK ? R1_FWD : R1_BCK;
  static constexpr int ZONE = (R0 + R1 + 1) / 2 * 2;
  static constexpr int TAB = 2 * N * P + N * T + N;   // per-thread-indexed table copy (stage C)
};

// PPT = quadrature points per thread: 2 (q0 and q0 + N/2 in turn) or 1 (twice the threads, fewer registers)
template <int K, int ZPC, int PPT = 2>
struct KB1V2Cfg {
  using Dm = V2Dims<K>;
  static constexpr int TPZ = Dm::N3 / PPT;                // threads per zone
  static constexpr int NTH = (ZPC * TPZ + 31) / 32 * 32;
  static constexpr int SMEM_DOUBLES = (Dm::TAB + 1) / 2 * 2 + 2 * ZPC * Dm::PFZ + ZPC * Dm::ZONE + 32;
  static constexpr int SMEM_BYTES = SMEM_DOUBLES * 8;
  static constexpr int IDS = (ZPC * Dm::P3 + NTH - 1) / NTH;   // node ids a thread prefetches per batch
};

__device__ __forceinline__ void cp_async8(void *dst, const void *src, bool valid) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(valid ? 8 : 0));
}
__device__ __forceinline__ void cp_async4(void *dst, const void *src) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(d), "l"(src));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int NPEND>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(NPEND)); }

// EX = 6: the point evaluation's lean eigen-solve (pointwise.cuh sym3_min_eig_lean, alpha folded into sigma)
template <int K, int ZPC, int MINB, int PPT = 2, int EX = 0>
__global__ void __launch_bounds__(KB1V2Cfg<K, ZPC, PPT>::NTH, MINB) kb1_v2_3d(const KB1Args a) {
  using Dm = V2Dims<K>;
  using C = CT<K>;
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, P2 = Dm::P2, P3 = Dm::P3, T2 = Dm::T2, T3 = Dm::T3;
  constexpr int N2 = Dm::N2, N3 = Dm::N3, NH = N / 2;
  constexpr int TPZ = KB1V2Cfg<K, ZPC, PPT>::TPZ;
  constexpr int NTH = KB1V2Cfg<K, ZPC, PPT>::NTH;
  static_assert(PPT == 1 || PPT == 2, "kb1_v2: one or two points per thread");
  static_assert(NTH <= 512, "block_min and the dt-filter slot share sRed[0, 32)");
  constexpr int IDS = KB1V2Cfg<K, ZPC, PPT>::IDS;
  extern __shared__ double smem[];
  double *sTab = smem;                               // B[N][P] G[N][P] Phi[N][T] W[N]
  double *sPF = smem + (Dm::TAB + 1) / 2 * 2;        // [2][ZPC][PFZ]
  double *sZone = sPF + 2 * ZPC * Dm::PFZ;           // [ZPC][ZONE]
  double *sRed = sZone + ZPC * Dm::ZONE;

  const int tid0 = threadIdx.x;
  const int64_t Z = a.num_zones, nn = a.num_nodes;
  const int64_t nb = (Z + ZPC - 1) / ZPC;            // zone batches; CTA c runs batches c, c+G, c+2G, ...
  const int64_t G = gridDim.x;

  // ---- a0: the gather, software-pipelined one batch ahead with cp.async --------------------------
  // ids[] holds the node ids of the batch whose copies are issued next (loaded one iteration earlier).
  int32_t ids[IDS];
  auto load_ids = [&](int64_t b, int tid) {
#pragma unroll
    for (int u = 0; u < IDS; ++u) {
      const int i = tid + u * NTH;
      const int zl = i / P3;
      const int64_t z = b * ZPC + zl;
      ids[u] = (i < ZPC * P3 && b < nb && z < Z) ? __ldg(a.zone_nodes + b * ZPC * P3 + i) : -1;
    }
  };
  auto issue = [&](int64_t b, double *pf, int tid) {
    if (b < nb) {
#pragma unroll
      for (int u = 0; u < IDS; ++u) {
        const int i = tid + u * NTH;
        if (i < ZPC * P3) {
          const int zl = i / P3, r = i - zl * P3;
          const bool v = ids[u] >= 0;
          const int64_t node = v ? ids[u] : 0;
          double *X = pf + zl * Dm::PFZ + Dm::PF_X + r;
#pragma unroll
          for (int c = 0; c < 3; ++c) {
            cp_async8(X + c * P3, a.x + c * nn + node, v);
            cp_async8(X + (3 + c) * P3, a.v + c * nn + node, v);
          }
        }
      }
      for (int i = tid; i < ZPC * (T3 + N3 + 10); i += NTH) {
        const int zl = i / (T3 + N3 + 10), r = i - zl * (T3 + N3 + 10);
        const int64_t z = b * ZPC + zl;
        const bool v = z < Z;
        const int64_t zz = v ? z : 0;
        double *dst = pf + zl * Dm::PFZ + Dm::PF_E + r;
        const double *src = r < T3 ? a.e + zz * T3 + r
                          : r < T3 + N3 ? a.rho0detJ0 + zz * N3 + (r - T3)
                          : r < T3 + N3 + 9 ? a.J0inv + zz * 9 + (r - T3 - N3) : a.zone_gamma + zz;
        cp_async8(dst, src, v);
      }
    }
    cp_async_commit();
  };

  for (int i = tid0; i < Dm::TAB; i += NTH) sTab[i] = __ldg(a.tab + i);
  if (threadIdx.x == 0) sRed[16] = 0.0;   // dt filter: the CTA's best exact inverse dt (block_min uses sRed[0, 8))
  int64_t b = blockIdx.x;
  load_ids(b, tid0);
  issue(b, sPF, tid0);
  load_ids(b + G, tid0);
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;

  for (int it = 0; b < nb; b += G, ++it) {
  // re-read the thread index every batch: keeps the compiler from hoisting all per-stage index and
  // address arithmetic out of the batch loop (which would pin ~100 registers and spill)
  int tid;
  asm volatile("mov.u32 %0, %%tid.x;" : "=r"(tid));
  const int cur = it & 1;
  double *PFc = sPF + cur * ZPC * Dm::PFZ;
  issue(b + G, sPF + (cur ^ 1) * ZPC * Dm::PFZ, tid);
  load_ids(b + 2 * G, tid);
  cp_async_wait<1>();
  __syncthreads();
  const int64_t zone0 = b * ZPC;

  // ---- stage A: a2 -> q2 for all slabs (values and derivatives); e: j2 -> q2 ---------------------
  for (int i = tid; i < ZPC * (6 * P2 + T2); i += NTH) {
    const int zl = i / (6 * P2 + T2), r = i - zl * (6 * P2 + T2);
    double *R0 = sZone + zl * Dm::ZONE;
    const double *pf = PFc + zl * Dm::PFZ;
    if (r < 6 * P2) {
      const int f = r / P2, aa = r - f * P2;
      double xv[P];
#pragma unroll
      for (int a2 = 0; a2 < P; ++a2) xv[a2] = pf[Dm::PF_X + f * P3 + a2 * P2 + aa];
      double *TB = R0 + Dm::O_T + (f * 2 + 0) * N * P2 + aa;
      double *TG = R0 + Dm::O_T + (f * 2 + 1) * N * P2 + aa;
#pragma unroll
      for (int q2 = 0; q2 < N; ++q2) {
        double tb = 0.0, tg = 0.0;
#pragma unroll
        for (int a2 = 0; a2 < P; ++a2) {
          tb = fma(C::B(q2, a2), xv[a2], tb);
          tg = fma(C::G(q2, a2), xv[a2], tg);
        }
        TB[q2 * P2] = tb;
        TG[q2 * P2] = tg;
      }
    } else {
      const int jj = r - 6 * P2;
      double ev[T];
#pragma unroll
      for (int j2 = 0; j2 < T; ++j2) ev[j2] = pf[Dm::PF_E + j2 * T2 + jj];
#pragma unroll
      for (int q2 = 0; q2 < N; ++q2) {
        double te = 0.0;
#pragma unroll
        for (int j2 = 0; j2 < T; ++j2) te = fma(C::Phi(q2, j2), ev[j2], te);
        R0[Dm::O_TE + q2 * T2 + jj] = te;
      }
    }
  }
  __syncthreads();

  // ---- stage B: a1 -> q1 --------------------------------------------------------------------------
  for (int i = tid; i < ZPC * (6 * N * P + N * T); i += NTH) {
    const int zl = i / (6 * N * P + N * T), r = i - zl * (6 * N * P + N * T);
    const double *R0 = sZone + zl * Dm::ZONE;
    double *R1 = sZone + zl * Dm::ZONE + Dm::R0;
    if (r < 6 * N * P) {
      const int f = r / (N * P), r2 = r - f * (N * P);
      const int q2 = r2 / P, a0 = r2 - q2 * P;
      double tb[P], tg[P];
#pragma unroll
      for (int a1 = 0; a1 < P; ++a1) {
        tb[a1] = R0[Dm::O_T + ((f * 2 + 0) * N + q2) * P2 + a1 * P + a0];
        tg[a1] = R0[Dm::O_T + ((f * 2 + 1) * N + q2) * P2 + a1 * P + a0];
      }
      double *U0 = R1 + Dm::O_U + (((f * 3 + 0) * N + q2) * N) * P + a0;
      double *U1 = R1 + Dm::O_U + (((f * 3 + 1) * N + q2) * N) * P + a0;
      double *U2 = R1 + Dm::O_U + (((f * 3 + 2) * N + q2) * N) * P + a0;
#pragma unroll
      for (int q1 = 0; q1 < N; ++q1) {
        double u0 = 0.0, u1 = 0.0, u2 = 0.0;
#pragma unroll
        for (int a1 = 0; a1 < P; ++a1) {
          u0 = fma(C::B(q1, a1), tb[a1], u0);
          u1 = fma(C::G(q1, a1), tb[a1], u1);
          u2 = fma(C::B(q1, a1), tg[a1], u2);
        }
        U0[q1 * P] = u0;
        U1[q1 * P] = u1;
        U2[q1 * P] = u2;
      }
    } else {
      const int r2 = r - 6 * N * P;
      const int q2 = r2 / T, j0 = r2 - q2 * T;
      double te[T];
#pragma unroll
      for (int j1 = 0; j1 < T; ++j1) te[j1] = R0[Dm::O_TE + q2 * T2 + j1 * T + j0];
#pragma unroll
      for (int q1 = 0; q1 < N; ++q1) {
        double ue = 0.0;
#pragma unroll
        for (int j1 = 0; j1 < T; ++j1) ue = fma(C::Phi(q1, j1), te[j1], ue);
        R1[Dm::O_UE + (q2 * N + q1) * T + j0] = ue;
      }
    }
  }
  __syncthreads();

  // ---- stage C (a0 -> q0) + point evaluation, two points per thread (q0 and q0 + N/2) ---------------
  // S/Pq of the first point go to R0 (free since stage B); those of the second are held in registers
  // across a barrier and written over U in R1 once every thread has finished reading U.
  const int my_zl = tid / TPZ, pr = tid - my_zl * TPZ;
  const bool has_point = my_zl < ZPC;
  const int64_t my_z = zone0 + my_zl;
  const bool active = has_point && my_z < Z;
  // PPT 2: points (q0a, q1, q2) and (q0a + N/2, q1, q2);  PPT 1: the point (q0a + hsel N/2, q1, q2)
  const int q0a = PPT == 2 ? pr % NH : (pr % N) % NH, hsel = PPT == 2 ? 0 : (pr % N) / NH;
  const int q1 = PPT == 2 ? (pr / NH) % N : (pr / N) % N, q2 = PPT == 2 ? pr / (NH * N) : pr / N2;
  double SB[10];
  if (has_point) {
    double *Rz = sZone + my_zl * Dm::ZONE;
    const double *R1 = Rz + Dm::R0;
    const double *pfz = PFc + my_zl * Dm::PFZ;
    const double *J0i = pfz + Dm::PF_J;
    const double gamma = J0i[9];
    const double *sW = sTab + 2 * N * P + N * T;
#pragma unroll 1
    for (int hh = 0; hh < PPT; ++hh) {
      const int h = PPT == 2 ? hh : hsel;
      const int q0 = q0a + h * NH;
      double g[18];
#pragma unroll
      for (int i = 0; i < 18; ++i) g[i] = 0.0;
#pragma unroll
      for (int a0 = 0; a0 < P; ++a0) {
        const double b = sTab[q0 * P + a0], gg = sTab[N * P + q0 * P + a0];
#pragma unroll
        for (int f = 0; f < 6; ++f)
#pragma unroll
          for (int m = 0; m < 3; ++m)
            g[f * 3 + m] = fma(m == 0 ? gg : b, R1[Dm::O_U + (((f * 3 + m) * N + q2) * N + q1) * P + a0], g[f * 3 + m]);
      }
      double eq = 0.0;
#pragma unroll
      for (int j0 = 0; j0 < T; ++j0) eq = fma(sTab[2 * N * P + q0 * T + j0], R1[Dm::O_UE + (q2 * N + q1) * T + j0], eq);
      double Jm[3][3], Gv[3][3];
#pragma unroll
      for (int c = 0; c < 3; ++c)
#pragma unroll
        for (int d = 0; d < 3; ++d) { Jm[c][d] = g[c * 3 + d]; Gv[c][d] = g[9 + c * 3 + d]; }
      const int q = (q2 * N + q1) * N + q0;
      const double R = active ? pfz[Dm::PF_R + q] : 1.0;
      const double alpha = sW[q0] * sW[q1] * sW[q2];
      PointOut<3> o;
      {   // dt filter (pointwise.cuh): exact sigma_min(J) only where a point can beat the CTA's best inverse dt
        const unsigned vm = __activemask();
        const double best = sRed[16];
        point_eval3<true, 0, EX>(Jm, Gv, eq, R, alpha, gamma, J0i, a.ph, o, best, vm);
        if (active && o.inv > best)
          atomicMax(reinterpret_cast<unsigned long long *>(sRed + 16), (unsigned long long)__double_as_longlong(o.inv));
      }
      if (h == 0) {
        double *SA = Rz + Dm::O_SA + (q2 * N + q1) * NH + q0a;
#pragma unroll
        for (int cd = 0; cd < 9; ++cd) SA[cd * N2 * NH] = o.S[cd / 3][cd % 3];
        SA[9 * N2 * NH] = o.P;
      } else {
#pragma unroll
        for (int cd = 0; cd < 9; ++cd) SB[cd] = o.S[cd / 3][cd % 3];
        SB[9] = o.P;
      }
      if (a.Sq != nullptr && active) {
#pragma unroll
        for (int cd = 0; cd < 9; ++cd) a.Sq[(my_z * N3 + q) * 9 + cd] = o.S[cd / 3][cd % 3];
      }
      if (active) {
        dtmin = fmin(dtmin, o.dt);
        bad |= o.bad;
      }
    }
  }
  __syncthreads();   // every U read is done
  if (has_point && (PPT == 2 || hsel == 1)) {
    double *SBp = sZone + my_zl * Dm::ZONE + Dm::R0 + Dm::O_SB + (q2 * N + q1) * NH + q0a;
#pragma unroll
    for (int cd = 0; cd < 10; ++cd) SBp[cd * N2 * NH] = SB[cd];
  }
  __syncthreads();

  // ---- stage C^T: q0 -> a0 ---------------------------------------------------------------------------
  for (int i = tid; i < ZPC * (3 * N2 + N2); i += NTH) {
    const int zl = i / (4 * N2), r = i - zl * (4 * N2);
    const double *SA = sZone + zl * Dm::ZONE + Dm::O_SA;
    double *R1 = sZone + zl * Dm::ZONE + Dm::R0;
    const double *SBr = R1 + Dm::O_SB;
    if (r < 3 * N2) {
      const int c = r / N2, col = r - c * N2;   // col = q2*N + q1
      double s0[N], s1[N], s2[N];
#pragma unroll
      for (int q0 = 0; q0 < N; ++q0) {
        const double *src = (q0 < NH ? SA : SBr) + col * NH + (q0 % NH);
        s0[q0] = src[(c * 3 + 0) * N2 * NH];
        s1[q0] = src[(c * 3 + 1) * N2 * NH];
        s2[q0] = src[(c * 3 + 2) * N2 * NH];
      }
#pragma unroll
      for (int a0 = 0; a0 < P; ++a0) {
        double y0 = 0.0, y1 = 0.0, y2 = 0.0;
#pragma unroll
        for (int q0 = 0; q0 < N; ++q0) {
          y0 = fma(C::G(q0, a0), s0[q0], y0);
          y1 = fma(C::B(q0, a0), s1[q0], y1);
          y2 = fma(C::B(q0, a0), s2[q0], y2);
        }
        R1[Dm::O_Y + ((c * 3 + 0) * P + a0) * N2 + col] = y0;
        R1[Dm::O_Y + ((c * 3 + 1) * P + a0) * N2 + col] = y1;
        R1[Dm::O_Y + ((c * 3 + 2) * P + a0) * N2 + col] = y2;
      }
    } else {
      const int col = r - 3 * N2;
      double pv[N];
#pragma unroll
      for (int q0 = 0; q0 < N; ++q0) pv[q0] = ((q0 < NH ? SA : SBr) + col * NH + (q0 % NH))[9 * N2 * NH];
#pragma unroll
      for (int j0 = 0; j0 < T; ++j0) {
        double y = 0.0;
#pragma unroll
        for (int q0 = 0; q0 < N; ++q0) y = fma(C::Phi(q0, j0), pv[q0], y);
        R1[Dm::O_YE + j0 * N2 + col] = y;
      }
    }
  }
  __syncthreads();

  // ---- stage B^T: q1 -> a1 ---------------------------------------------------------------------------
  for (int i = tid; i < ZPC * (3 * P * N + T * N); i += NTH) {
    const int zl = i / (3 * P * N + T * N), r = i - zl * (3 * P * N + T * N);
    double *R0 = sZone + zl * Dm::ZONE;                 // Z out
    const double *R1 = sZone + zl * Dm::ZONE + Dm::R0;  // Y in
    if (r < 3 * P * N) {
      const int c = r / (P * N), r2 = r - c * (P * N);
      const int a0 = r2 / N, q2 = r2 - a0 * N;
      double y0[N], y1[N], y2[N];
#pragma unroll
      for (int q1 = 0; q1 < N; ++q1) {
        y0[q1] = R1[Dm::O_Y + ((c * 3 + 0) * P + a0) * N2 + q2 * N + q1];
        y1[q1] = R1[Dm::O_Y + ((c * 3 + 1) * P + a0) * N2 + q2 * N + q1];
        y2[q1] = R1[Dm::O_Y + ((c * 3 + 2) * P + a0) * N2 + q2 * N + q1];
      }
#pragma unroll
      for (int a1 = 0; a1 < P; ++a1) {
        double zb = 0.0, zg = 0.0;
#pragma unroll
        for (int q1 = 0; q1 < N; ++q1) {
          zb = fma(C::B(q1, a1), y0[q1], zb);
          zb = fma(C::G(q1, a1), y1[q1], zb);
          zg = fma(C::B(q1, a1), y2[q1], zg);
        }
        R0[Dm::O_Z + ((c * 2 + 0) * N + q2) * P2 + a1 * P + a0] = zb;
        R0[Dm::O_Z + ((c * 2 + 1) * N + q2) * P2 + a1 * P + a0] = zg;
      }
    } else {
      const int r2 = r - 3 * P * N;
      const int j0 = r2 / N, q2 = r2 - j0 * N;
      double ye[N];
#pragma unroll
      for (int q1 = 0; q1 < N; ++q1) ye[q1] = R1[Dm::O_YE + j0 * N2 + q2 * N + q1];
#pragma unroll
      for (int j1 = 0; j1 < T; ++j1) {
        double ze = 0.0;
#pragma unroll
        for (int q1 = 0; q1 < N; ++q1) ze = fma(C::Phi(q1, j1), ye[q1], ze);
        R0[Dm::O_ZE + q2 * T2 + j1 * T + j0] = ze;
      }
    }
  }
  __syncthreads();

  // ---- stage A^T: q2 -> a2, straight to global --------------------------------------------------------
  for (int i = tid; i < ZPC * (3 * P2 + T2); i += NTH) {
    const int zl = i / (3 * P2 + T2), r = i - zl * (3 * P2 + T2);
    const int64_t z = zone0 + zl;
    const double *R0 = sZone + zl * Dm::ZONE;
    if (z >= Z) continue;
    if (r < 3 * P2) {
      const int c = r / P2, aa = r - c * P2;
      double zb[N], zg[N];
#pragma unroll
      for (int q2 = 0; q2 < N; ++q2) {
        zb[q2] = R0[Dm::O_Z + ((c * 2 + 0) * N + q2) * P2 + aa];
        zg[q2] = R0[Dm::O_Z + ((c * 2 + 1) * N + q2) * P2 + aa];
      }
#pragma unroll
      for (int a2 = 0; a2 < P; ++a2) {
        double s = 0.0;
#pragma unroll
        for (int q2 = 0; q2 < N; ++q2) {
          s = fma(C::B(q2, a2), zb[q2], s);
          s = fma(C::G(q2, a2), zg[q2], s);
        }
        a.Fz1[(z * 3 + c) * P3 + a2 * P2 + aa] = s;
      }
    } else {
      const int jj = r - 3 * P2;
      double ze[N];
#pragma unroll
      for (int q2 = 0; q2 < N; ++q2) ze[q2] = R0[Dm::O_ZE + q2 * T2 + jj];
#pragma unroll
      for (int j2 = 0; j2 < T; ++j2) {
        double s = 0.0;
#pragma unroll
        for (int q2 = 0; q2 < N; ++q2) s = fma(C::Phi(q2, j2), ze[q2], s);
        a.FTv[z * T3 + j2 * T2 + jj] = s;
      }
    }
  }
  }   // batches
  cp_async_wait<0>();
  if (bad) dtmin = 0.0;
  const double m = block_min(dtmin, sRed);
  if (tid0 == 0) a.cta_dt[blockIdx.x] = m;
}
