// KB1 v3 — 3D corner force with the sum-factorized contractions on the FP64 tensor path (DMMA).
//
// Same mathematics and shared-memory plan as kb1_v2.cuh (eq (4)-(6); DESIGN.md §1 rows
// a0-a5), but every contraction whose outputs go to shared memory — the forward stages A (a2 -> q2)
// and B (a1 -> q1) and the back stages C^T, B^T, A^T — runs as warp-level FP64 matrix products
// (mma.sync.m8n8k4.f64 -> DMMA.8x8x4; tcgen05 has no FP64 kind on sm_100a).  Each 1-D table is an
// A operand held in registers for the whole stage (no per-FMA constant loads), the data matrix is the B
// operand gathered from shared memory (one load per lane per k-step for 256 FMAs of the warp), and the
// accumulators go straight to their shared-memory layout.  Stage C (a0 -> q0), whose outputs feed
// the per-point physics in registers, stays on DFMA (thread = point).
//
// Tiles: rows (the output index) in blocks of 8, the contraction index in steps of 4 (zero padded:
// p = k+1 = 5 -> 8 for k = 4), columns (the batch of 1-D lines) in blocks of 8.
#pragma once
#include "kb1_v2.cuh"

__device__ __forceinline__ void dmma(double &d0, double &d1, double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
      : "+d"(d0), "+d"(d1)
      : "d"(a), "d"(b));
}

// A-operand fragment of a 1-D table tab[q][a] (row stride `ld`, valid nq x na):
// forward (rows = q, k = a) or transposed (rows = a, k = q).
template <bool TRANS>
__device__ __forceinline__ double tfrag(const double *tab, int ld, int nq, int na, int m, int k) {
  const int q = TRANS ? k : m, a = TRANS ? m : k;
  return (q < nq && a < na) ? tab[q * ld + a] : 0.0;
}

template <int K>
struct V3Dims : V2Dims<K> {
  using B_ = V2Dims<K>;
  static constexpr int N = B_::N, P = B_::P, T = B_::T, P2 = B_::P2, P3 = B_::P3, T2 = B_::T2, T3 = B_::T3;
  static constexpr int N2 = B_::N2, N3 = B_::N3, NH = B_::NH, SH = B_::SH;
  // R0: X[6][P^3] E[T^3] T[6][2][N][P^2] TE[N][T^2]  ->  S/Pq (q0 < N/2)  ->  Z ZE
  static constexpr int O_X = 0, O_E = 6 * P3, O_T = O_E + T3, O_TE = O_T + 12 * N * P2;
  static constexpr int R0_FWD = O_TE + N * T2;
  static constexpr int O_SA = 0, O_Z = 0, O_ZE = 6 * N * P2, R0_Z = O_ZE + N * T2;
  static constexpr int R0 = R0_FWD > SH ? (R0_FWD > R0_Z ? R0_FWD : R0_Z) : (SH > R0_Z ? SH : R0_Z);
  static constexpr int R1 = B_::R1;
  static constexpr int O_U = B_::O_U, O_UE = B_::O_UE, O_SB = B_::O_SB, O_Y = B_::O_Y, O_YE = B_::O_YE;
  static constexpr int ZONE = (R0 + R1 + 10 + 1) / 2 * 2;   // + J0^{-1}, gamma
  static constexpr int TAB = B_::TAB;
  // tile counts
  static constexpr int MT_N = (N + 7) / 8, MT_P = (P + 7) / 8, MT_T = (T + 7) / 8;
  static constexpr int KS_P = (P + 3) / 4, KS_N = (N + 3) / 4, KS_T = (T + 3) / 4;
};

template <int K, int ZPC>
struct KB1V3Cfg {
  using Dm = V3Dims<K>;
  static constexpr int NTH = (ZPC * Dm::TPZ + 31) / 32 * 32;
  static constexpr int NW = NTH / 32;
  static constexpr int SMEM_DOUBLES = (Dm::TAB + 1) / 2 * 2 + ZPC * Dm::ZONE + 32;
  static constexpr int SMEM_BYTES = SMEM_DOUBLES * 8;
};

template <int K, int ZPC, int MINB>
__global__ void __launch_bounds__(KB1V3Cfg<K, ZPC>::NTH, MINB) kb1_v3_3d(const KB1Args a) {
  using Dm = V3Dims<K>;
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, P2 = Dm::P2, P3 = Dm::P3, T2 = Dm::T2, T3 = Dm::T3;
  constexpr int N2 = Dm::N2, N3 = Dm::N3, TPZ = Dm::TPZ, NH = Dm::NH;
  constexpr int NTH = KB1V3Cfg<K, ZPC>::NTH, NW = KB1V3Cfg<K, ZPC>::NW;
  static_assert(NTH <= 512, "block_min and the dt-filter slot share sRed[0, 32)");
  constexpr int MT_N = Dm::MT_N, MT_P = Dm::MT_P, MT_T = Dm::MT_T, KS_P = Dm::KS_P, KS_N = Dm::KS_N, KS_T = Dm::KS_T;
  extern __shared__ double smem[];
  double *sTab = smem;                                  // B[N][P] G[N][P] Phi[N][T] W[N]
  const double *tB = sTab, *tG = sTab + N * P, *tPhi = sTab + 2 * N * P, *sW = sTab + 2 * N * P + N * T;
  double *sZone = smem + (Dm::TAB + 1) / 2 * 2;       // [ZPC][ZONE]
  double *sRed = sZone + ZPC * Dm::ZONE;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  int nstamp = 0;
#define KB1_STAMP()                                                                       \
  do {                                                                                    \
    if (a.prof != nullptr && tid == 0) a.prof[blockIdx.x * 16 + nstamp] = clock64();      \
    ++nstamp;                                                                             \
  } while (0)
  KB1_STAMP();
  const int lr = lane >> 2, lc = lane & 3;              // fragment row / k-column of this lane
  const int64_t zone0 = (int64_t)blockIdx.x * ZPC;
  const int64_t Z = a.num_zones, nn = a.num_nodes;

  // ---- a0: tables, gather ----------------------------------------------------------------------
  for (int i = tid; i < Dm::TAB; i += NTH) sTab[i] = __ldg(a.tab + i);
  if (threadIdx.x == 0) sRed[16] = 0.0;   // dt filter: the CTA's best exact inverse dt (block_min uses sRed[0, 8))
  {   // rho0|J0| of this thread's two points is read in the point stage: start the DRAM fetches into L1 now
    const int zl = tid / Dm::TPZ, pr = tid - zl * Dm::TPZ;
    if (zl < ZPC && zone0 + zl < Z) {
      const int q = ((pr / (Dm::N / 2 * Dm::N)) * Dm::N + (pr / (Dm::N / 2)) % Dm::N) * Dm::N + pr % (Dm::N / 2);
      const double *Rq = a.rho0detJ0 + (zone0 + zl) * Dm::N3 + q;
      asm volatile("prefetch.global.L1 [%0];" ::"l"(Rq));
      asm volatile("prefetch.global.L1 [%0];" ::"l"(Rq + Dm::N / 2));
    }
  }
  for (int i = tid; i < ZPC * P3; i += NTH) {
    const int zl = i / P3, r = i - zl * P3;
    const int64_t z = zone0 + zl;
    double *X = sZone + zl * Dm::ZONE + Dm::O_X;
    double vals[6] = {0, 0, 0, 0, 0, 0};
    if (z < Z) {
      const int64_t node = __ldg(a.zone_nodes + z * P3 + r);
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        vals[c] = __ldg(a.x + c * nn + node);
        vals[3 + c] = __ldg(a.v + c * nn + node);
      }
    }
#pragma unroll
    for (int f = 0; f < 6; ++f) X[f * P3 + r] = vals[f];
  }
  for (int i = tid; i < ZPC * T3; i += NTH) {
    const int zl = i / T3, r = i - zl * T3;
    const int64_t z = zone0 + zl;
    sZone[zl * Dm::ZONE + Dm::O_E + r] = (z < Z) ? __ldg(a.e + z * T3 + r) : 0.0;
  }
  for (int i = tid; i < ZPC * 10; i += NTH) {
    const int zl = i / 10, r = i - zl * 10;
    const int64_t z = zone0 + zl;
    double val;
    if (r < 9) val = (z < Z) ? __ldg(a.J0inv + z * 9 + r) : (r % 4 == 0 ? 1.0 : 0.0);
    else val = (z < Z) ? __ldg(a.zone_gamma + z) : 1.4;
    sZone[zl * Dm::ZONE + Dm::R0 + Dm::R1 + r] = val;
  }
  __syncthreads();
  KB1_STAMP();

  // Index clamping instead of bounds tests: a padded k (or column) reads a valid neighbour whose A-fragment
  // coefficient is zero (or whose output is discarded), so every B-fragment load is unconditional.
  static_assert(MT_N == 1 && MT_P == 1 && MT_T == 1, "kb1_v3 tiles rows into one block of 8 (k <= 4)");
  // forward table fragments (rows = lane >> 2, k-column = 4s + (lane & 3)), live through stages A and B only
  double fB[KS_P], fG[KS_P], fP[KS_T];
#pragma unroll
  for (int s = 0; s < KS_P; ++s) {
    fB[s] = tfrag<false>(tB, P, N, P, lr, 4 * s + lc);
    fG[s] = tfrag<false>(tG, P, N, P, lr, 4 * s + lc);
  }
#pragma unroll
  for (int s = 0; s < KS_T; ++s) fP[s] = tfrag<false>(tPhi, T, N, T, lr, 4 * s + lc);

  // ---- stage A: T_m[f][q2][aa] = sum_a2 M[q2][a2] X[f][a2][aa]  (M = B, G);  TE = Phi . E --------------
  {
    constexpr int NC = 6 * P2, NTL = (NC + 7) / 8, NCE = T2, NTE = (NCE + 7) / 8, PER = NTL + NTE;
    for (int j = warp; j < ZPC * PER; j += NW) {
      const int zl = j / PER, tl = j - zl * PER;
      double *R0 = sZone + zl * Dm::ZONE;
      if (tl < NTL) {
        const int nb = min(tl * 8 + lr, NC - 1);          // this lane's B column (clamped)
        const int fb = nb / P2, ab_ = nb - fb * P2;
        const double *Xb = R0 + Dm::O_X + fb * P3 + ab_;
        double db0 = 0.0, db1 = 0.0, dg0 = 0.0, dg1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_P; ++s) {
          const double b = Xb[min(4 * s + lc, P - 1) * P2];
          dmma(db0, db1, fB[s], b);
          dmma(dg0, dg1, fG[s], b);
        }
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = tl * 8 + 2 * lc + i;
          if (lr < N && n < NC) {
            const int f = n / P2, aa = n - f * P2;
            R0[Dm::O_T + (f * 2 + 0) * N * P2 + lr * P2 + aa] = i ? db1 : db0;
            R0[Dm::O_T + (f * 2 + 1) * N * P2 + lr * P2 + aa] = i ? dg1 : dg0;
          }
        }
      } else {
        const int te = tl - NTL;
        const int nb = min(te * 8 + lr, NCE - 1);
        double d0 = 0.0, d1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_T; ++s) dmma(d0, d1, fP[s], R0[Dm::O_E + min(4 * s + lc, T - 1) * T2 + nb]);
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = te * 8 + 2 * lc + i;
          if (lr < N && n < NCE) R0[Dm::O_TE + lr * T2 + n] = i ? d1 : d0;
        }
      }
    }
  }
  __syncthreads();
  KB1_STAMP();

  // ---- stage B: U0 = B.TB, U1 = G.TB, U2 = B.TG over a1 -> q1 (columns (f, q2, a0)); UE = Phi.TE --------
  {
    constexpr int NC = 6 * N * P, NTL = (NC + 7) / 8, NCE = N * T, NTE = (NCE + 7) / 8, PER = NTL + NTE;
    for (int j = warp; j < ZPC * PER; j += NW) {
      const int zl = j / PER, tl = j - zl * PER;
      const double *R0 = sZone + zl * Dm::ZONE;
      double *R1 = sZone + zl * Dm::ZONE + Dm::R0;
      if (tl < NTL) {
        const int nb = min(tl * 8 + lr, NC - 1);
        const int fb = nb / (N * P), rb = nb - fb * (N * P), q2b = rb / P, a0b = rb - q2b * P;
        const double *TBb = R0 + Dm::O_T + ((fb * 2 + 0) * N + q2b) * P2 + a0b;
        const double *TGb = TBb + N * P2;
        double u00 = 0.0, u01 = 0.0, u10 = 0.0, u11 = 0.0, u20 = 0.0, u21 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_P; ++s) {
          const int a1 = min(4 * s + lc, P - 1);
          const double tb = TBb[a1 * P], tg = TGb[a1 * P];
          dmma(u00, u01, fB[s], tb);
          dmma(u10, u11, fG[s], tb);
          dmma(u20, u21, fB[s], tg);
        }
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = tl * 8 + 2 * lc + i;
          if (lr < N && n < NC) {
            const int f = n / (N * P), rr = n - f * (N * P), q2 = rr / P, a0 = rr - q2 * P;
            double *U = R1 + Dm::O_U + (((f * 3) * N + q2) * N + lr) * P + a0;
            U[0] = i ? u01 : u00;
            U[N2 * P] = i ? u11 : u10;
            U[2 * N2 * P] = i ? u21 : u20;
          }
        }
      } else {
        const int te = tl - NTL;
        const int nb = min(te * 8 + lr, NCE - 1);
        const int q2b = nb / T, j0b = nb - q2b * T;
        double d0 = 0.0, d1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_T; ++s) dmma(d0, d1, fP[s], R0[Dm::O_TE + q2b * T2 + min(4 * s + lc, T - 1) * T + j0b]);
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = te * 8 + 2 * lc + i;
          if (lr < N && n < NCE) {
            const int q2 = n / T, j0 = n - q2 * T;
            R1[Dm::O_UE + (q2 * N + lr) * T + j0] = i ? d1 : d0;
          }
        }
      }
    }
  }
  __syncthreads();
  KB1_STAMP();

  // ---- stage C (a0 -> q0, DFMA) + point evaluation, two points per thread --------------------------
  const int my_zl = tid / TPZ, pr = tid - my_zl * TPZ;
  const bool has_point = my_zl < ZPC;
  const int64_t my_z = zone0 + my_zl;
  const bool active = has_point && my_z < Z;
  const int q0a = pr % NH, q1 = (pr / NH) % N, q2 = pr / (NH * N);
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;
  double SB[10];
  if (has_point) {
    double *Rz = sZone + my_zl * Dm::ZONE;
    const double *R1 = Rz + Dm::R0;
    const double *J0i = Rz + Dm::R0 + Dm::R1;
    const double gamma = J0i[9];
#pragma unroll 1
    for (int h = 0; h < 2; ++h) {
      const int q0 = q0a + h * NH;
      double g[18];
#pragma unroll
      for (int i = 0; i < 18; ++i) g[i] = 0.0;
#pragma unroll
      for (int a0 = 0; a0 < P; ++a0) {
        const double b = tB[q0 * P + a0], gg = tG[q0 * P + a0];
#pragma unroll
        for (int f = 0; f < 6; ++f)
#pragma unroll
          for (int m = 0; m < 3; ++m)
            g[f * 3 + m] = fma(m == 0 ? gg : b, R1[Dm::O_U + (((f * 3 + m) * N + q2) * N + q1) * P + a0], g[f * 3 + m]);
      }
      double eq = 0.0;
#pragma unroll
      for (int j0 = 0; j0 < T; ++j0) eq = fma(tPhi[q0 * T + j0], R1[Dm::O_UE + (q2 * N + q1) * T + j0], eq);
      double Jm[3][3], Gv[3][3];
#pragma unroll
      for (int c = 0; c < 3; ++c)
#pragma unroll
        for (int d = 0; d < 3; ++d) { Jm[c][d] = g[c * 3 + d]; Gv[c][d] = g[9 + c * 3 + d]; }
      const int q = (q2 * N + q1) * N + q0;
      const double R = active ? __ldg(a.rho0detJ0 + my_z * N3 + q) : 1.0;
      const double alpha = sW[q0] * sW[q1] * sW[q2];
      PointOut<3> o;
      {   // dt filter (pointwise.cuh): exact sigma_min(J) only where a point can beat the CTA's best inverse dt
        const unsigned vm = __activemask();
        const double best = sRed[16];
        point_eval3<true>(Jm, Gv, eq, R, alpha, gamma, J0i, a.ph, o, best, vm);
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
  __syncthreads();
  KB1_STAMP();   // every U read is done
  if (has_point) {
    double *SBp = sZone + my_zl * Dm::ZONE + Dm::R0 + Dm::O_SB + (q2 * N + q1) * NH + q0a;
#pragma unroll
    for (int cd = 0; cd < 10; ++cd) SBp[cd * N2 * NH] = SB[cd];
  }
  __syncthreads();
  KB1_STAMP();

  // transposed table fragments for the back stages (reloaded here: not kept live through the point stage)
  double fBt[KS_N], fGt[KS_N], fPt[KS_N];
#pragma unroll
  for (int s = 0; s < KS_N; ++s) {
    fBt[s] = tfrag<true>(tB, P, N, P, lr, 4 * s + lc);
    fGt[s] = tfrag<true>(tG, P, N, P, lr, 4 * s + lc);
    fPt[s] = tfrag<true>(tPhi, T, N, T, lr, 4 * s + lc);
  }

  // ---- stage C^T: Y[cd][a0][col] = sum_q0 M[q0][a0] S_cd[q0][col] (M = G for d = 0 else B), col = (q2,q1);
  //      YE[j0][col] = sum_q0 Phi[q0][j0] Pq[q0][col]  (10 "matrices" x N^2 columns) -------------------------
  {
    constexpr int NTL = (N2 + 7) / 8, PER = 10 * NTL, JOBS = ZPC * PER;
    for (int j = warp; j < JOBS; j += NW) {
      const int zl = j / PER, jr = j - zl * PER;
      const int cd = jr / NTL, tl = jr - cd * NTL;
      const double *SA = sZone + zl * Dm::ZONE + Dm::O_SA + cd * N2 * NH;
      double *R1 = sZone + zl * Dm::ZONE + Dm::R0;
      const double *SBr = R1 + Dm::O_SB + cd * N2 * NH;
      const int colb = min(tl * 8 + lr, N2 - 1);
      double d0 = 0.0, d1 = 0.0;
#pragma unroll
      for (int s = 0; s < KS_N; ++s) {
        const int q0 = min(4 * s + lc, N - 1);
        const double b = (q0 < NH ? SA : SBr)[colb * NH + (q0 % NH)];
        dmma(d0, d1, cd == 9 ? fPt[s] : (cd % 3 == 0 ? fGt[s] : fBt[s]), b);
      }
#pragma unroll
      for (int i = 0; i < 2; ++i) {
        const int col = tl * 8 + 2 * lc + i;
        if (col < N2) {
          if (cd < 9 && lr < P) R1[Dm::O_Y + (cd * P + lr) * N2 + col] = i ? d1 : d0;
          if (cd == 9 && lr < T) R1[Dm::O_YE + lr * N2 + col] = i ? d1 : d0;
        }
      }
    }
  }
  __syncthreads();
  KB1_STAMP();

  // ---- stage B^T: ZB[c][q2][a1][a0] = sum_q1 B[q1][a1] Y_c0 + G[q1][a1] Y_c1 ; ZG = sum_q1 B[q1][a1] Y_c2
  //      (columns (q2, a0)); ZE[q2][j1][j0] = sum_q1 Phi[q1][j1] YE[j0][q2][q1] (columns (q2, j0)) --------
  {
    constexpr int NC = N * P, NTL = (NC + 7) / 8, NCE = N * T, NTE = (NCE + 7) / 8, PER = 3 * NTL + NTE;
    for (int j = warp; j < ZPC * PER; j += NW) {
      const int zl = j / PER, jr = j - zl * PER;
      double *R0 = sZone + zl * Dm::ZONE;
      const double *R1 = sZone + zl * Dm::ZONE + Dm::R0;
      if (jr < 3 * NTL) {
        const int c = jr / NTL, tl = jr - c * NTL;
        const int nb = min(tl * 8 + lr, NC - 1);
        const int q2b = nb / P, a0b = nb - q2b * P;
        const double *Yb = R1 + Dm::O_Y + (c * 3 * P + a0b) * N2 + q2b * N;
        double zb0 = 0.0, zb1 = 0.0, zg0 = 0.0, zg1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_N; ++s) {
          const int q1 = min(4 * s + lc, N - 1);
          dmma(zb0, zb1, fBt[s], Yb[q1]);
          dmma(zb0, zb1, fGt[s], Yb[P * N2 + q1]);
          dmma(zg0, zg1, fBt[s], Yb[2 * P * N2 + q1]);
        }
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = tl * 8 + 2 * lc + i;
          if (lr < P && n < NC) {
            const int q2 = n / P, a0 = n - q2 * P;
            R0[Dm::O_Z + ((c * 2 + 0) * N + q2) * P2 + lr * P + a0] = i ? zb1 : zb0;
            R0[Dm::O_Z + ((c * 2 + 1) * N + q2) * P2 + lr * P + a0] = i ? zg1 : zg0;
          }
        }
      } else {
        const int te = jr - 3 * NTL;
        const int nb = min(te * 8 + lr, NCE - 1);
        const int q2b = nb / T, j0b = nb - q2b * T;
        double d0 = 0.0, d1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_N; ++s) dmma(d0, d1, fPt[s], R1[Dm::O_YE + j0b * N2 + q2b * N + min(4 * s + lc, N - 1)]);
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = te * 8 + 2 * lc + i;
          if (lr < T && n < NCE) {
            const int q2 = n / T, j0 = n - q2 * T;
            R0[Dm::O_ZE + q2 * T2 + lr * T + j0] = i ? d1 : d0;
          }
        }
      }
    }
  }
  __syncthreads();
  KB1_STAMP();

  // ---- stage A^T: F_c[a2][aa] = sum_q2 B[q2][a2] ZB_c[q2][aa] + G[q2][a2] ZG_c[q2][aa] -> global;
  //      FTv[j2][jj] = sum_q2 Phi[q2][j2] ZE[q2][jj] -> global ------------------------------------------
  {
    constexpr int NTL = (P2 + 7) / 8, NTE = (T2 + 7) / 8, PER = 3 * NTL + NTE;
    for (int j = warp; j < ZPC * PER; j += NW) {
      const int zl = j / PER, jr = j - zl * PER;
      const int64_t z = zone0 + zl;
      const double *R0 = sZone + zl * Dm::ZONE;
      if (jr < 3 * NTL) {
        const int c = jr / NTL, tl = jr - c * NTL;
        const int nb = min(tl * 8 + lr, P2 - 1);
        const double *Zb = R0 + Dm::O_Z + c * 2 * N * P2 + nb;
        double d0 = 0.0, d1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_N; ++s) {
          const int q2 = min(4 * s + lc, N - 1);
          dmma(d0, d1, fBt[s], Zb[q2 * P2]);
          dmma(d0, d1, fGt[s], Zb[(N + q2) * P2]);
        }
        if (z < Z && lr < P) {
#pragma unroll
          for (int i = 0; i < 2; ++i) {
            const int n = tl * 8 + 2 * lc + i;
            if (n < P2) a.Fz1[(z * 3 + c) * P3 + lr * P2 + n] = i ? d1 : d0;
          }
        }
      } else {
        const int te = jr - 3 * NTL;
        const int nb = min(te * 8 + lr, T2 - 1);
        double d0 = 0.0, d1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_N; ++s) dmma(d0, d1, fPt[s], R0[Dm::O_ZE + min(4 * s + lc, N - 1) * T2 + nb]);
        if (z < Z && lr < T) {
#pragma unroll
          for (int i = 0; i < 2; ++i) {
            const int n = te * 8 + 2 * lc + i;
            if (n < T2) a.FTv[z * T3 + lr * T2 + n] = i ? d1 : d0;
          }
        }
      }
    }
  }
  if (bad) dtmin = 0.0;
  const double m = block_min(dtmin, sRed);
  if (tid == 0) a.cta_dt[blockIdx.x] = m;
  KB1_STAMP();
#undef KB1_STAMP
}
