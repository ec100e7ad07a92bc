// KB1 v8 — 3D corner force for high orders (5 <= k <= 8, C5 is k = 8): one zone per CTA, q2 slabs,
// contraction stages register-blocked with the 1-D tables as constant-bank operands.
//
// Same mathematics and slab order as kb1_corner_force_3d (eq (4)-(6); DESIGN.md §1 rows a0-a5):
// the whole-zone intermediates of k = 8 (U alone would be 330 KB) do not fit in shared memory, so the
// zone is processed in N = 2k slabs of fixed q2.  What changes is the shape of every contraction stage.
// ncu on the v1 kernel (profiles/r01_kb1_c5_ncu.txt) showed the shared-memory pipe at 87 % of peak: each
// FMA of a stage read its table coefficient and its operand from shared memory.  Here each work item
// loads its operand line once and produces a whole output line from it, with the table coefficients
// taken from the constant bank at compile-time indices (uniform LDCU feeding DFMA's uniform-register
// operand; the offset `o` is 0 but loop-variant so the loads are not hoisted out of the slab loop):
//   A   (a2 -> q2 of slab q2):  item (f, a1 a0): 9 loads -> 2 outputs     (table row q2: uniform)
//   B   (a1 -> q1):             item (f, m, a0): 9 loads -> 16 outputs    (was 36 loads per 3 FMAs)
//   C   (a0 -> q0) + point:     thread (q0, q1): U rows padded to 16-byte pairs, 16-byte loads
//   C^T (q0 -> a0):             item (c d, q1):  8 x 16-byte loads -> 9 outputs, warp-uniform table
//   B^T (q1 -> a1):             item (c, a0):    16-32 loads -> 9 outputs, one warp per table pattern
//   A^T (q2 -> a2, accumulate): item (c, a1 a0): 2 loads -> 9 accumulators (table row q2: uniform)
// S is stored with rows of N + 2 doubles so the C^T row loads (16 bytes, 8 consecutive rows per phase)
// are conflict-free.  Two CTAs per SM (111 KB of shared memory each at k = 8).
#pragma once
#include "kb1_v6.cuh"

template <int K>
struct V8Dims {
  static constexpr int N = 2 * K, P = K + 1, T = K;
  static constexpr int P2 = P * P, NK = P * P * P, NT = T * T * T, NS = N * N, T2 = T * T;
  static constexpr int PP = (P + 1) / 2 * 2;           // U row stride (16-byte pairs)
  static constexpr int SR = N + 2;                     // S row stride (conflict-free 16-byte row loads)
  // Phi rows padded to TS = T + 1 doubles in shared memory: the point stage reads Phi[q0][j] with q0 per lane,
  // and a row stride of T = 8 doubles put 16 lanes on 2 sixteen-byte slots (8-way; ncu on C5)
  static constexpr int TS = T + 1;
  static constexpr int TAB = (2 * N * P + N * TS + N + 1) / 2 * 2;
  static constexpr int O_X = 0, O_E = 6 * NK, O_AF = O_E + NT, O_AE = O_AF + 3 * NK, O_J0 = O_AE + NT;
  static constexpr int FIX = (O_J0 + 10 + 1) / 2 * 2;
  // region A: T (TB, TG [6][P2] each, TE [T2]) -> S [10][N][SR] -> Z (ZB, ZG [3][P2] each, ZE [T2])
  static constexpr int A_T = 12 * P2 + T2, A_S = 10 * N * SR, A_Z = 6 * P2 + T2;
  static constexpr int RA = ((A_T > A_S ? A_T : A_S) > A_Z ? (A_T > A_S ? A_T : A_S) : A_Z);
  // region B: U [6][3][N][PP] + UE [N][T] -> Y [3][3][N][P] + YE [T][N]
  static constexpr int B_U = 18 * N * PP + N * T, B_Y = 9 * N * P + T * N;
  static constexpr int RB = B_U > B_Y ? B_U : B_Y;
  static constexpr int OFF_FIX = TAB, OFF_A = OFF_FIX + FIX, OFF_B = OFF_A + (RA + 1) / 2 * 2;
  static constexpr int OFF_RED = OFF_B + (RB + 1) / 2 * 2;
  static constexpr int TOTAL = OFF_RED + 32;
};

template <int K>
struct KB1V8Cfg {
  using Dm = V8Dims<K>;
  static constexpr int NTH = (Dm::NS + 31) / 32 * 32;
  static constexpr int SMEM_BYTES = Dm::TOTAL * 8;
};

template <int K, int MINB>
__global__ void __launch_bounds__(KB1V8Cfg<K>::NTH, MINB) kb1_v8_3d(const KB1Args a) {
  using Dm = V8Dims<K>;
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, P2 = Dm::P2, NK = Dm::NK, NT = Dm::NT, NS = Dm::NS;
  constexpr int T2 = Dm::T2, PP = Dm::PP, SR = Dm::SR;
  constexpr int NTH = KB1V8Cfg<K>::NTH;
  constexpr bool FILTER = NS % 32 == 0;   // every warp full of points: the dt filter's vote is legal
  static_assert(NTH >= 192, "stage C^T: six warps of row items (k >= 7)");
  static_assert(NTH >= 6 * 3 * P + T, "stage B: one item per thread");
  static_assert(NTH >= 3 * P2, "stage A^T: one item per thread");
  extern __shared__ double smem[];
  double *sB = smem, *sG = sB + N * P, *sPhi = sG + N * P, *sW = sPhi + N * Dm::TS;
  double *sF = smem + Dm::OFF_FIX;
  double *sX = sF + Dm::O_X, *sE = sF + Dm::O_E, *sAF = sF + Dm::O_AF, *sAE = sF + Dm::O_AE, *sJ0 = sF + Dm::O_J0;
  double *sA = smem + Dm::OFF_A, *sBr = smem + Dm::OFF_B, *sRed = smem + Dm::OFF_RED;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t z = blockIdx.x;                  // one zone per CTA (grid = Z)
  const int64_t nn = a.num_nodes;

  // ---- a0: tables + gather ----------------------------------------------------------------------
  for (int i = tid; i < 2 * N * P + N * T + N; i += NTH) {   // B, G; Phi into rows of TS; W
    const double t = __ldg(a.tab + i);
    if (i < 2 * N * P) smem[i] = t;
    else if (i < 2 * N * P + N * T) sPhi[((i - 2 * N * P) / T) * Dm::TS + (i - 2 * N * P) % T] = t;
    else sW[i - 2 * N * P - N * T] = t;
  }
  for (int r = tid; r < NK; r += NTH) {
    const int64_t node = __ldg(a.zone_nodes + z * NK + r);
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      sX[c * NK + r] = __ldg(a.x + c * nn + node);
      sX[(3 + c) * NK + r] = __ldg(a.v + c * nn + node);
      sAF[c * NK + r] = 0.0;
    }
  }
  for (int r = tid; r < NT; r += NTH) {
    sE[r] = __ldg(a.e + z * NT + r);
    sAE[r] = 0.0;
  }
  if (tid < 9) sJ0[tid] = __ldg(a.J0inv + z * 9 + tid);
  if (tid == 9) sJ0[9] = __ldg(a.zone_gamma + z);
  if (tid == 0) sRed[8] = 0.0;   // dt filter: the CTA's best exact inverse dt
  __syncthreads();

  const int q0 = tid % N, q1 = tid / N;
  const bool has_point = tid < NS;
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;

#pragma unroll 1
  for (int q2 = 0; q2 < N; ++q2) {
    const int o = a.zero * (q2 + 1);   // 0, but loop-variant and uniform: the table loads stay here
    // rho0|J0| of this thread's point of slab q2 is read in the point stage: start its DRAM fetch into L1
    // now, two stages ahead (ncu on v8: long_scoreboard was the second stall reason, profiles/r01_kb1_c5_default_ncu)
    if (has_point)
      asm volatile("prefetch.global.L1 [%0];" ::"l"(a.rho0detJ0 + z * (int64_t)(N * NS) + (q2 * N + q1) * N + q0));
    // ---- stage A: a2 -> q2 (TB, TG of the 6 fields; TE) -------------------------------------------
    {
      const CTZ<K> C{o};
#pragma unroll
      for (int rd = 0; rd < (6 * P2 + T2 + NTH - 1) / NTH; ++rd) {
        const int r = tid + rd * NTH;
        if (r < 6 * P2) {
          const int f = r / P2, rr = r - f * P2;
          double tb = 0.0, tg = 0.0;
#pragma unroll
          for (int a2 = 0; a2 < P; ++a2) {
            const double xv = sX[f * NK + a2 * P2 + rr];
            tb = fma(C.B(q2, a2), xv, tb);
            tg = fma(C.G(q2, a2), xv, tg);
          }
          sA[f * P2 + rr] = tb;
          sA[6 * P2 + f * P2 + rr] = tg;
        } else if (r < 6 * P2 + T2) {
          const int jj = r - 6 * P2;
          double te = 0.0;
#pragma unroll
          for (int j2 = 0; j2 < T; ++j2) te = fma(C.Phi(q2, j2), sE[j2 * T2 + jj], te);
          sA[12 * P2 + jj] = te;
        }
      }
    }
    __syncthreads();
    // ---- stage B: a1 -> q1; item (f, m, a0) produces U[f][m][q1 = 0..N-1][a0] ----------------------
    {
      const CTZ<K> C{2 * o};
      const int r = tid;
      if (r < 18 * P) {
        const int fm = r / P, a0 = r - fm * P, f = fm / 3, m = fm - f * 3;
        const double *src = sA + (m == 2 ? 6 * P2 : 0) + f * P2 + a0;   // TG for m = 2, else TB
        double tv[P];
#pragma unroll
        for (int a1 = 0; a1 < P; ++a1) tv[a1] = src[a1 * P];
        double *U = sBr + fm * N * PP + a0;
        if (m == 1) {
#pragma unroll
          for (int qq1 = 0; qq1 < N; ++qq1) {
            double u = 0.0;
#pragma unroll
            for (int a1 = 0; a1 < P; ++a1) u = fma(C.G(qq1, a1), tv[a1], u);
            U[qq1 * PP] = u;
          }
        } else {
#pragma unroll
          for (int qq1 = 0; qq1 < N; ++qq1) {
            double u = 0.0;
#pragma unroll
            for (int a1 = 0; a1 < P; ++a1) u = fma(C.B(qq1, a1), tv[a1], u);
            U[qq1 * PP] = u;
          }
        }
        if (P < PP) {   // zero pad of the 16-byte pairs (read by stage C's paired loads, coefficient 0)
#pragma unroll
          for (int qq1 = 0; qq1 < N; ++qq1)
            if (a0 == P - 1) U[qq1 * PP + 1] = 0.0;
        }
      } else if (r < 18 * P + T) {
        const int j0 = r - 18 * P;
        double tv[T];
#pragma unroll
        for (int j1 = 0; j1 < T; ++j1) tv[j1] = sA[12 * P2 + j1 * T + j0];
#pragma unroll
        for (int qq1 = 0; qq1 < N; ++qq1) {
          double u = 0.0;
#pragma unroll
          for (int j1 = 0; j1 < T; ++j1) u = fma(C.Phi(qq1, j1), tv[j1], u);
          sBr[18 * N * PP + qq1 * T + j0] = u;
        }
      }
    }
    __syncthreads();
    // ---- stage C (a0 -> q0) + point evaluation ------------------------------------------------------
    if (has_point) {
      double g18[18];
#pragma unroll
      for (int i = 0; i < 18; ++i) g18[i] = 0.0;
#pragma unroll
      for (int pa = 0; pa < PP / 2; ++pa) {
        const int a0 = 2 * pa;
        const double b0 = sB[q0 * P + a0], g0 = sG[q0 * P + a0];
        const double b1 = a0 + 1 < P ? sB[q0 * P + a0 + 1] : 0.0, g1 = a0 + 1 < P ? sG[q0 * P + a0 + 1] : 0.0;
#pragma unroll
        for (int fm = 0; fm < 18; ++fm) {
          double u0, u1;
          lds_f64x2(sBr + (fm * N + q1) * PP + a0, u0, u1);
          const bool dx = fm % 3 == 0;
          g18[fm] = fma(dx ? g0 : b0, u0, g18[fm]);
          g18[fm] = fma(dx ? g1 : b1, u1, g18[fm]);
        }
      }
      double eq = 0.0;
#pragma unroll
      for (int j0 = 0; j0 < T; ++j0) eq = fma(sPhi[q0 * Dm::TS + j0], sBr[18 * N * PP + q1 * T + j0], eq);
      double Jm[3][3], Gv[3][3];
#pragma unroll
      for (int c = 0; c < 3; ++c)
#pragma unroll
        for (int d = 0; d < 3; ++d) { Jm[c][d] = g18[c * 3 + d]; Gv[c][d] = g18[9 + c * 3 + d]; }
      const int q = (q2 * N + q1) * N + q0;
      const double R = __ldg(a.rho0detJ0 + z * (int64_t)(N * NS) + q);
      const double alpha = sW[q0] * sW[q1] * sW[q2];
      PointOut<3> pt;
      if (FILTER) {
        const double best = sRed[8];
        point_eval3<true>(Jm, Gv, eq, R, alpha, sJ0[9], sJ0, a.ph, pt, best);
        double mi = pt.inv;
#pragma unroll
        for (int s = 16; s > 0; s >>= 1) mi = fmax(mi, __shfl_xor_sync(0xffffffffu, mi, s));
        if (lane == 0 && mi > best)
          atomicMax(reinterpret_cast<unsigned long long *>(sRed + 8), (unsigned long long)__double_as_longlong(mi));
      } else {
        point_eval3(Jm, Gv, eq, R, alpha, sJ0[9], sJ0, a.ph, pt);
      }
      double *S = sA + q1 * SR + q0;
#pragma unroll
      for (int cd = 0; cd < 9; ++cd) S[cd * N * SR] = pt.S[cd / 3][cd % 3];
      S[9 * N * SR] = pt.P;
      if (a.Sq != nullptr) {
#pragma unroll
        for (int cd = 0; cd < 9; ++cd) a.Sq[(z * (int64_t)(N * NS) + q) * 9 + cd] = pt.S[cd / 3][cd % 3];
      }
      dtmin = fmin(dtmin, pt.dt);
      bad |= pt.bad;
    }
    __syncthreads();
    // ---- stage C^T: q0 -> a0; warps 0-1: d = 0 components (G), 2-4: d != 0 (B), 5: Pq (Phi) ---------
    {
      const CTZ<K> C{3 * o};
      const int grp = warp < 2 ? 0 : warp < 5 ? 1 : warp < 6 ? 2 : 3;
      const int li = (warp - (grp == 0 ? 0 : grp == 1 ? 2 : 5)) * 32 + lane;   // index inside the group
      const int cdi = li / N, qq1 = li - cdi * N;
      int cd = -1;
      if (grp == 0 && cdi < 3) cd = cdi * 3;                         // 0, 3, 6
      if (grp == 1 && cdi < 6) cd = (cdi / 2) * 3 + 1 + (cdi & 1);   // 1, 2, 4, 5, 7, 8
      if (grp == 2 && cdi < 1) cd = 9;
      if (cd >= 0 && qq1 < N) {
        double sv[N];
        const double *row = sA + (cd * N + qq1) * SR;
#pragma unroll
        for (int pq = 0; pq < N / 2; ++pq) lds_f64x2(row + 2 * pq, sv[2 * pq], sv[2 * pq + 1]);
        if (grp == 0) {
#pragma unroll
          for (int a0 = 0; a0 < P; ++a0) {
            double y = 0.0;
#pragma unroll
            for (int qq0 = 0; qq0 < N; ++qq0) y = fma(C.G(qq0, a0), sv[qq0], y);
            sBr[(cd * N + qq1) * P + a0] = y;
          }
        } else if (grp == 1) {
#pragma unroll
          for (int a0 = 0; a0 < P; ++a0) {
            double y = 0.0;
#pragma unroll
            for (int qq0 = 0; qq0 < N; ++qq0) y = fma(C.B(qq0, a0), sv[qq0], y);
            sBr[(cd * N + qq1) * P + a0] = y;
          }
        } else {
#pragma unroll
          for (int j0 = 0; j0 < T; ++j0) {
            double y = 0.0;
#pragma unroll
            for (int qq0 = 0; qq0 < N; ++qq0) y = fma(C.Phi(qq0, j0), sv[qq0], y);
            sBr[9 * N * P + j0 * N + qq1] = y;
          }
        }
      }
    }
    __syncthreads();
    // ---- stage B^T: q1 -> a1; warp 0: ZB items (c, a0), warp 1: ZG items, warp 2: ZE items (j0) -----
    {
      const CTZ<K> C{4 * o};
      if (warp == 0 && lane < 3 * P) {
        const int c = lane / P, a0 = lane - c * P;
        const double *y0 = sBr + ((c * 3 + 0) * N) * P + a0, *y1 = sBr + ((c * 3 + 1) * N) * P + a0;
        double v0[N], v1[N];
#pragma unroll
        for (int qq1 = 0; qq1 < N; ++qq1) { v0[qq1] = y0[qq1 * P]; v1[qq1] = y1[qq1 * P]; }
#pragma unroll
        for (int a1 = 0; a1 < P; ++a1) {
          double s = 0.0;
#pragma unroll
          for (int qq1 = 0; qq1 < N; ++qq1) {
            s = fma(C.B(qq1, a1), v0[qq1], s);
            s = fma(C.G(qq1, a1), v1[qq1], s);
          }
          sA[c * P2 + a1 * P + a0] = s;
        }
      } else if (warp == 1 && lane < 3 * P) {
        const int c = lane / P, a0 = lane - c * P;
        const double *y2 = sBr + ((c * 3 + 2) * N) * P + a0;
        double v2[N];
#pragma unroll
        for (int qq1 = 0; qq1 < N; ++qq1) v2[qq1] = y2[qq1 * P];
#pragma unroll
        for (int a1 = 0; a1 < P; ++a1) {
          double s = 0.0;
#pragma unroll
          for (int qq1 = 0; qq1 < N; ++qq1) s = fma(C.B(qq1, a1), v2[qq1], s);
          sA[3 * P2 + c * P2 + a1 * P + a0] = s;
        }
      } else if (warp == 2 && lane < T) {
        const int j0 = lane;
        double ve[N];
#pragma unroll
        for (int qq1 = 0; qq1 < N; ++qq1) ve[qq1] = sBr[9 * N * P + j0 * N + qq1];
#pragma unroll
        for (int j1 = 0; j1 < T; ++j1) {
          double s = 0.0;
#pragma unroll
          for (int qq1 = 0; qq1 < N; ++qq1) s = fma(C.Phi(qq1, j1), ve[qq1], s);
          sA[6 * P2 + j1 * T + j0] = s;
        }
      }
    }
    __syncthreads();
    // ---- stage A^T: accumulate q2 -> a2; item (c, a1 a0) owns 9 accumulators, e items on the top ---
    {
      const CTZ<K> C{5 * o};
      if (tid < 3 * P2) {
        const int c = tid / P2, rr = tid - c * P2;
        const double zb = sA[c * P2 + rr], zg = sA[3 * P2 + c * P2 + rr];
        double *acc = sAF + c * NK + rr;
#pragma unroll
        for (int a2 = 0; a2 < P; ++a2) acc[a2 * P2] = fma(C.B(q2, a2), zb, fma(C.G(q2, a2), zg, acc[a2 * P2]));
      }
      if (tid >= NTH - T2) {
        const int jj = tid - (NTH - T2);
        const double ze = sA[6 * P2 + jj];
#pragma unroll
        for (int j2 = 0; j2 < T; ++j2) sAE[j2 * T2 + jj] = fma(C.Phi(q2, j2), ze, sAE[j2 * T2 + jj]);
      }
    }
    __syncthreads();   // region A (Z) is overwritten by the next slab's stage A
  }
  // ---- outputs ----------------------------------------------------------------------------------
  for (int i = tid; i < 3 * NK; i += NTH) a.Fz1[z * 3 * NK + i] = sAF[i];
  for (int i = tid; i < NT; i += NTH) a.FTv[z * NT + i] = sAE[i];
  if (bad) dtmin = 0.0;
  const double m = block_min(dtmin, sRed);
  if (tid == 0) a.cta_dt[blockIdx.x] = m;
}
