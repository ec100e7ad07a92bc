// KB1 v5 — warp-specialized 3D corner force (k <= 4) with the Jacobian's last contraction on DMMA.
//
// Same mathematics as kb1_v3.cuh / kb1_v4.cuh (eq (4)-(6); DESIGN.md §1 rows a0-a5) and the
// same two-group pipeline as v4 (point warps PW on zone i, DMMA warps KW on zones i-1 and i+1, one CTA
// barrier per zone).  What moved (profiles/r01_kb1_c4_v4 source view: PW was the critical path, its
// stage C — 94 DFMA + 45 shared loads per point — 30 % of PW's samples, while KW sat 41 % at barriers):
//
//   * stage C of the three POSITION fields (a0 -> q0 for x: the 9 entries of J) runs in KW as DMMA
//     (data as the A operand, the 1-D table as the B operand, so a lane's two accumulators are two
//     neighbouring q0 of one (q2, q1) line and leave as one 16-byte shared store);
//   * J lands in the "JS" buffer [10][N^3]; the point warps read it and write S = alpha sigma adj(J)^T
//     and S : grad^v back IN PLACE (same thread, same point slots: no hazard), which is the buffer the
//     back stages read — so U and S no longer need separate double buffers;
//   * rho0|J0|(q) of the next zone is staged into shared memory by cp.async together with the gather
//     (PW no longer issues global loads).
// PW keeps stage C of the velocity fields (grad^v) and e(q), then the point physics of pointwise.cuh.
#pragma once
#include "kb1_v4.cuh"

template <int K>
struct V5Dims {
  static constexpr int N = 2 * K, P = K + 1, T = K;
  static constexpr int P2 = P * P, P3 = P * P * P, T2 = T * T, T3 = T * T * T, N2 = N * N, N3 = N * N * N;
  static constexpr int NH = N / 2, TPZ = N3 / 2;
  static constexpr int TAB = (2 * N * P + N * T + N + 1) / 2 * 2;
  // UV buffer (KW -> PW): velocity-field U[3][3][N][N][P], UE[N][N][T], R = rho0|J0| [N^3]
  static constexpr int O_UE = 9 * N2 * P, O_R = (O_UE + N2 * T + 1) / 2 * 2, UVBUF = (O_R + N3 + 1) / 2 * 2;
  // JS buffer (KW -> PW -> KW): J[9][N^3] in, S[9][N^3] + Pq[N^3] out (in place)
  static constexpr int O_PQ = 9 * N3, JSBUF = 10 * N3;
  // KW scratch: XE (X[6][P^3] E[T^3] J0[9] gamma, cp.async) | forward T/TE + UX | back Y/YE + Z/ZE
  static constexpr int XE_X = 0, XE_E = 6 * P3, XE_J = XE_E + T3, XE = (XE_J + 10 + 1) / 2 * 2;
  static constexpr int O_T = 0, O_TE = 12 * N * P2, O_UX = (O_TE + N * T2 + 1) / 2 * 2, FWREG = O_UX + 9 * N2 * P;
  // Y / YE rows (one per (component, a0) / j0) are YS = N^2 + 4 apart: kb1_v10's DMMA C^T stores and B^T
  // loads put 5 rows in one warp access, which a stride of N^2 = 64 maps onto the same banks (5-way)
  static constexpr int YS = N2 + 4;
  static constexpr int O_Y = 0, O_YE = 9 * P * YS, O_Z = O_YE + T * YS, O_ZE = O_Z + 6 * N * P2;
  static constexpr int YZREG = O_ZE + N * T2;
  static constexpr int WREG = ((FWREG > YZREG ? FWREG : YZREG) + 1) / 2 * 2;
  // totals (every region starts on a 16-byte boundary)
  static constexpr int OFF_JS = TAB, OFF_UV = OFF_JS + 2 * JSBUF, OFF_XE = OFF_UV + 2 * UVBUF, OFF_W = OFF_XE + XE;
  static constexpr int OFF_J = OFF_W + WREG;            // J0^{-1} + gamma for the two buffers [2][10]
  static constexpr int OFF_RED = OFF_J + 20;
  static constexpr int OFF_ID = OFF_RED + 32;          // zone -> node ids of the next two zones, int32 [2][P^3]
  static constexpr int OFF_MB = OFF_ID + (2 * P3 + 1) / 2;   // two mbarriers (kb1_v10.cuh bulk copies)
  static constexpr int OFF_XEB = OFF_MB + 2;                  // second XE buffer (kb1_v10.cuh PWG)
  static constexpr int TOTAL = OFF_XEB + XE;
  static constexpr int MT = (N + 7) / 8, KS_P = (P + 3) / 4, KS_N = (N + 3) / 4, KS_T = (T + 3) / 4;
};

// MODE picks the register split between the point warps and the DMMA warps (setmaxnreg) and the DMMA
// tiles in flight per warp: 0 = 168 / 88 / 8, 1 = 184 / 72 / 4, 2 = 200 / 56 / 2, 3 = 176 / 80 / 4, 4 = 160 / 96 / 8.
template <int K, int MODE = 0>
struct KB1V5Cfg {
  using Dm = V5Dims<K>;
  static constexpr int NPW = (Dm::N3 / 2 + 127) / 128 * 128;   // 2 points per point-thread
  static constexpr int NKW = 256;
  static constexpr int NTH = NPW + NKW;
  static constexpr int REG_PW = MODE == 0 ? 168 : MODE == 1 ? 184 : MODE == 2 ? 200 : MODE == 3 ? 176 : 160;
  static constexpr int REG_KW = MODE == 0 ? 88 : MODE == 1 ? 72 : MODE == 2 ? 56 : MODE == 3 ? 80 : 96;
  static constexpr int KWCH = MODE == 0 ? 8 : MODE == 1 ? 4 : MODE == 2 ? 2 : MODE == 3 ? 4 : 8;   // DMMA tiles in flight per warp
  static constexpr int REG_LAUNCH = (65536 / NTH) / 8 * 8;
  static_assert(NPW * REG_PW + NKW * REG_KW <= NTH * REG_LAUNCH, "register split exceeds the CTA's allocation");
  static constexpr int SMEM_BYTES = Dm::TOTAL * 8;
};

__device__ __forceinline__ void sts_f64x2(double *dst, double a, double b) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("st.shared.v2.f64 [%0], {%1, %2};\n" ::"r"(d), "d"(a), "d"(b) : "memory");
}

// DIAG (timing experiments only, wrong results): 1 = the DMMA warps skip their stages, 2 = the point
// warps skip theirs; selected by name (BLAST_CF_KB1=v5.d1 / v5.d2), never by the autotuner.
template <int K, int DIAG = 0, int MODE = 0>
__global__ void __launch_bounds__(KB1V5Cfg<K, MODE>::NTH, 1) kb1_v5_3d(const KB1Args a) {
  using Dm = V5Dims<K>;
  using Cfg = KB1V5Cfg<K, MODE>;
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, P2 = Dm::P2, P3 = Dm::P3, T2 = Dm::T2, T3 = Dm::T3;
  constexpr int N2 = Dm::N2, N3 = Dm::N3, NH = Dm::NH, TPZ = Dm::TPZ;
  constexpr int KS_P = Dm::KS_P, KS_N = Dm::KS_N, KS_T = Dm::KS_T;
  constexpr int NPW = Cfg::NPW, NKW = Cfg::NKW, NKWW = NKW / 32, KWCH = Cfg::KWCH;
  static_assert(NKW >= P3, "the gather gives one node per DMMA-warp thread");
  static_assert(Dm::MT == 1, "kb1_v5: rows in one block of 8 (k <= 4)");
  static_assert(N == 8, "kb1_v5: the J tiles store two neighbouring q0 of a line of 8");
  extern __shared__ double smem[];
  double *sTab = smem;
  const double *tB = sTab, *tG = sTab + N * P, *tPhi = sTab + 2 * N * P, *sW = sTab + 2 * N * P + N * T;
  double *sJS = smem + Dm::OFF_JS, *sUV = smem + Dm::OFF_UV, *sXE = smem + Dm::OFF_XE, *sWk = smem + Dm::OFF_W;
  double *sJ = smem + Dm::OFF_J, *sRed = smem + Dm::OFF_RED;

  const int tid = threadIdx.x;
  const bool is_kw = tid >= NPW;
  const int ktid = tid - NPW;                       // KW thread index (valid if is_kw)
  const int64_t Z = a.num_zones, nn = a.num_nodes;
  const int64_t G = gridDim.x;
  const int64_t nz = Z > blockIdx.x ? (Z - 1 - blockIdx.x) / G + 1 : 0;   // zones of this CTA
  auto zone_of = [&](int64_t i) { return (int64_t)blockIdx.x + i * G; };
  // stage clocks of the DMMA warps (a.prof != nullptr only): sKP[s] accumulates the cycles of stage s,
  // sKP[15] holds the last stamp; written by KW thread 0 alone (PW's dt reduction uses sRed[0, 16))
  long long *sKP = reinterpret_cast<long long *>(smem + Dm::OFF_RED + 16);
  auto kstamp = [&](int slot) {
    if (a.prof != nullptr && threadIdx.x == NPW) {
      const long long t = clock64();
      sKP[slot] += t - sKP[15];
      sKP[15] = t;
    }
  };

  for (int i = tid; i < 2 * N * P + N * T + N; i += Cfg::NTH) sTab[i] = __ldg(a.tab + i);
  if (tid == 0) sRed[8] = 0.0;   // dt filter: best exact inverse dt of this CTA (point_eval3<true>)

  // ---------------- KW helpers ----------------
  // node ids travel by cp.async into shared memory one zone ahead (a register copy of an __ldg result
  // would be spilled by the 88-register warps and the spill store would wait for the load)
  int32_t *sID = reinterpret_cast<int32_t *>(smem + Dm::OFF_ID);
  auto kw_load_id = [&](int64_t i) {
    if (i < nz && ktid < P3) cp_async4(sID + (i & 1) * P3 + ktid, a.zone_nodes + zone_of(i) * P3 + ktid);
  };
  auto kw_issue = [&](int64_t i) {       // cp.async gather of zone i into XE and R of UV[i & 1]
    if (i < nz) {
      const int64_t z = zone_of(i);
      if (ktid < P3) {
        const int64_t node = sID[(i & 1) * P3 + ktid];
#pragma unroll
        for (int c = 0; c < 3; ++c) {
          cp_async8(sXE + Dm::XE_X + c * P3 + ktid, a.x + c * nn + node, true);
          cp_async8(sXE + Dm::XE_X + (3 + c) * P3 + ktid, a.v + c * nn + node, true);
        }
      }
      for (int r = ktid; r < T3 + 10; r += NKW) {
        const double *src = r < T3 ? a.e + z * T3 + r : r < T3 + 9 ? a.J0inv + z * 9 + (r - T3) : a.zone_gamma + z;
        cp_async8(sXE + Dm::XE_E + r, src, true);
      }
      double *R = sUV + (i & 1) * Dm::UVBUF + Dm::O_R;
      for (int r = ktid; r < N3; r += NKW) cp_async8(R + r, a.rho0detJ0 + z * N3 + r, true);
    }
  };
  // forward stages A, B (all fields) and C (position fields) of the zone in XE -> UV buffer ub, JS buffer jb
  auto kw_forward = [&](double *ub, double *jb, double *js) {
    const int ktid = opaque_tid() - NPW, kwarp = ktid >> 5, lr = (ktid & 31) >> 2, lc = ktid & 3;
    double fB[KS_P], fG[KS_P], fP[KS_T];
#pragma unroll
    for (int s = 0; s < KS_P; ++s) {
      fB[s] = tfrag<false>(tB, P, N, P, lr, 4 * s + lc);
      fG[s] = tfrag<false>(tG, P, N, P, lr, 4 * s + lc);
    }
#pragma unroll
    for (int s = 0; s < KS_T; ++s) fP[s] = tfrag<false>(tPhi, T, N, T, lr, 4 * s + lc);
    if (ktid < 10) js[ktid] = sXE[Dm::XE_J + ktid];
    double *Tr = sWk, *UX = sWk + Dm::O_UX;
    {   // stage A: T_M[f][q2][a1 a0] = sum_a2 M[q2][a2] X[f][a2][a1 a0], M = B, G
      constexpr int NC = 6 * P2, NTL = (NC + 7) / 8, JPWT = (NTL + NKWW - 1) / NKWW, JPW = JPWT < KWCH ? JPWT : KWCH;
      for (int t0 = 0; t0 < JPWT; t0 += JPW) {
        double bx[JPW][KS_P];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int nb = min((kwarp + (t0 + t) * NKWW) * 8 + lr, NC - 1);
          const int fb = nb / P2, ab_ = nb - fb * P2;
#pragma unroll
          for (int s = 0; s < KS_P; ++s) bx[t][s] = sXE[Dm::XE_X + fb * P3 + min(4 * s + lc, P - 1) * P2 + ab_];
        }
        double db[JPW][2], dg[JPW][2];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          db[t][0] = db[t][1] = dg[t][0] = dg[t][1] = 0.0;
#pragma unroll
          for (int s = 0; s < KS_P; ++s) {
            dmma(db[t][0], db[t][1], fB[s], bx[t][s]);
            dmma(dg[t][0], dg[t][1], fG[s], bx[t][s]);
          }
        }
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = kwarp + (t0 + t) * NKWW;
#pragma unroll
          for (int i = 0; i < 2; ++i) {
            const int n = j * 8 + 2 * lc + i;
            if (j < NTL && lr < N && n < NC) {
              const int f = n / P2, aa = n - f * P2;
              Tr[Dm::O_T + (f * 2 + 0) * N * P2 + lr * P2 + aa] = db[t][i];
              Tr[Dm::O_T + (f * 2 + 1) * N * P2 + lr * P2 + aa] = dg[t][i];
            }
          }
        }
      }
      constexpr int NCE = T2, NTE = (NCE + 7) / 8;   // TE = Phi . E
      for (int te = kwarp; te < NTE; te += NKWW) {
        const int nb = min(te * 8 + lr, NCE - 1);
        double d0 = 0.0, d1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_T; ++s) dmma(d0, d1, fP[s], sXE[Dm::XE_E + min(4 * s + lc, T - 1) * T2 + nb]);
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = te * 8 + 2 * lc + i;
          if (lr < N && n < NCE) Tr[Dm::O_TE + lr * T2 + n] = i ? d1 : d0;
        }
      }
    }
    kw_bar<NKW>();
    kstamp(8);
    {   // stage B: U0 = B.TB, U1 = G.TB, U2 = B.TG; position fields -> UX (KW scratch), velocity -> ub
      constexpr int NC = 6 * N * P, NTL = (NC + 7) / 8, JPWT = (NTL + NKWW - 1) / NKWW, JPW = JPWT < KWCH ? JPWT : KWCH;
      for (int t0 = 0; t0 < JPWT; t0 += JPW) {
        double tb[JPW][KS_P], tg[JPW][KS_P];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int nb = min((kwarp + (t0 + t) * NKWW) * 8 + lr, NC - 1);
          const int fb = nb / (N * P), rb = nb - fb * (N * P), q2b = rb / P, a0b = rb - q2b * P;
          const double *TBb = Tr + Dm::O_T + ((fb * 2 + 0) * N + q2b) * P2 + a0b;
#pragma unroll
          for (int s = 0; s < KS_P; ++s) {
            const int a1 = min(4 * s + lc, P - 1);
            tb[t][s] = TBb[a1 * P];
            tg[t][s] = TBb[N * P2 + a1 * P];
          }
        }
        double u[JPW][3][2];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
#pragma unroll
          for (int m = 0; m < 3; ++m) u[t][m][0] = u[t][m][1] = 0.0;
#pragma unroll
          for (int s = 0; s < KS_P; ++s) {
            dmma(u[t][0][0], u[t][0][1], fB[s], tb[t][s]);
            dmma(u[t][1][0], u[t][1][1], fG[s], tb[t][s]);
            dmma(u[t][2][0], u[t][2][1], fB[s], tg[t][s]);
          }
        }
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = kwarp + (t0 + t) * NKWW;
#pragma unroll
          for (int i = 0; i < 2; ++i) {
            const int n = j * 8 + 2 * lc + i;
            if (j < NTL && lr < N && n < NC) {
              const int f = n / (N * P), rr = n - f * (N * P), q2 = rr / P, a0 = rr - q2 * P;
              double *U = (f < 3 ? UX + f * 3 * N2 * P : ub + (f - 3) * 3 * N2 * P) + (q2 * N + lr) * P + a0;
              U[0] = u[t][0][i];
              U[N2 * P] = u[t][1][i];
              U[2 * N2 * P] = u[t][2][i];
            }
          }
        }
      }
      constexpr int NCE = N * T, NTE = (NCE + 7) / 8;   // UE = Phi . TE
      for (int te = kwarp; te < NTE; te += NKWW) {
        const int nb = min(te * 8 + lr, NCE - 1);
        const int q2b = nb / T, j0b = nb - q2b * T;
        double d0 = 0.0, d1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_T; ++s) dmma(d0, d1, fP[s], Tr[Dm::O_TE + q2b * T2 + min(4 * s + lc, T - 1) * T + j0b]);
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = te * 8 + 2 * lc + i;
          if (lr < N && n < NCE) {
            const int q2 = n / T, j0 = n - q2 * T;
            ub[Dm::O_UE + (q2 * N + lr) * T + j0] = i ? d1 : d0;
          }
        }
      }
    }
    kw_bar<NKW>();
    kstamp(9);
    {   // stage C (position fields): J[c][m][q2 q1][q0] = sum_a0 UX[c][m][q2 q1][a0] M_m[q0][a0]
        // A operand = UX (rows = 8 lines (q2, q1), k = a0), B operand = the table (k = a0, n = q0):
        // the B fragment of lane (lr, lc) is M[lr][4s + lc], the same registers as the A fragments above.
      constexpr int NTL = N2 / 8, NJ = 9 * NTL, JPWT = (NJ + NKWW - 1) / NKWW, JPW = JPWT < 5 ? JPWT : 5;
      for (int t0 = 0; t0 < JPWT; t0 += JPW) {
        double ux[JPW][KS_P];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = min(kwarp + (t0 + t) * NKWW, NJ - 1);
          const int cm = j / NTL, tl = j - cm * NTL;
          const double *Ub = UX + cm * N2 * P + (tl * 8 + lr) * P;
#pragma unroll
          for (int s = 0; s < KS_P; ++s) ux[t][s] = Ub[min(4 * s + lc, P - 1)];   // padded k: table entry is 0
        }
        double d[JPW][2];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = min(kwarp + (t0 + t) * NKWW, NJ - 1);
          const bool dx = (j / NTL) % 3 == 0;                // m = 0: d/dxi_0 uses G
          d[t][0] = d[t][1] = 0.0;
#pragma unroll
          for (int s = 0; s < KS_P; ++s) dmma(d[t][0], d[t][1], ux[t][s], dx ? fG[s] : fB[s]);
        }
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = kwarp + (t0 + t) * NKWW;
          if (j < NJ) {
            const int cm = j / NTL, tl = j - cm * NTL;
            sts_f64x2(jb + cm * N3 + (tl * 8 + lr) * N + 2 * lc, d[t][0], d[t][1]);
          }
        }
      }
    }
    kstamp(10);
  };
  // back stages C^T, B^T, A^T of zone z from the JS buffer sb (S[9][N^3], Pq[N^3])
  auto kw_back = [&](const double *sb, int64_t z) {
    const int ktid = opaque_tid() - NPW, kwarp = ktid >> 5, lr = (ktid & 31) >> 2, lc = ktid & 3;
    double fBt[KS_N], fGt[KS_N], fPt[KS_N];
#pragma unroll
    for (int s = 0; s < KS_N; ++s) {
      fBt[s] = tfrag<true>(tB, P, N, P, lr, 4 * s + lc);
      fGt[s] = tfrag<true>(tG, P, N, P, lr, 4 * s + lc);
      fPt[s] = tfrag<true>(tPhi, T, N, T, lr, 4 * s + lc);
    }
    double *Wr = sWk;
    {   // C^T: each warp takes one column tile (col = q2*N + q1), five matrices at a time
      constexpr int NTL = (N2 + 7) / 8;
      for (int tl = kwarp; tl < NTL; tl += NKWW) {
        const int colb = min(tl * 8 + lr, N2 - 1);
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          double sv[5][KS_N];
#pragma unroll
          for (int c5 = 0; c5 < 5; ++c5)
#pragma unroll
            for (int s = 0; s < KS_N; ++s) sv[c5][s] = sb[(h * 5 + c5) * N3 + colb * N + min(4 * s + lc, N - 1)];
          double d[5][2];
#pragma unroll
          for (int c5 = 0; c5 < 5; ++c5) {
            const int cd = h * 5 + c5;
            d[c5][0] = d[c5][1] = 0.0;
#pragma unroll
            for (int s = 0; s < KS_N; ++s)
              dmma(d[c5][0], d[c5][1], cd == 9 ? fPt[s] : (cd % 3 == 0 ? fGt[s] : fBt[s]), sv[c5][s]);
          }
#pragma unroll
          for (int i = 0; i < 2; ++i) {
            const int col = tl * 8 + 2 * lc + i;
            if (col < N2) {
#pragma unroll
              for (int c5 = 0; c5 < 5; ++c5) {
                const int cd = h * 5 + c5;
                if (cd < 9 && lr < P) Wr[Dm::O_Y + (cd * P + lr) * N2 + col] = d[c5][i];
                if (cd == 9 && lr < T) Wr[Dm::O_YE + lr * N2 + col] = d[c5][i];
              }
            }
          }
        }
      }
    }
    kw_bar<NKW>();
    kstamp(4);
    {   // B^T
      constexpr int NC = N * P, NTL = (NC + 7) / 8, NJ = 3 * NTL, JPWT = (NJ + NKWW - 1) / NKWW, JPW = JPWT < KWCH ? JPWT : KWCH;
      for (int t0 = 0; t0 < JPWT; t0 += JPW) {
        double y[JPW][3][KS_N];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = min(kwarp + (t0 + t) * NKWW, NJ - 1);
          const int c = j / NTL, tl = j - c * NTL;
          const int nb = min(tl * 8 + lr, NC - 1);
          const int q2b = nb / P, a0b = nb - q2b * P;
          const double *Yb = Wr + Dm::O_Y + (c * 3 * P + a0b) * N2 + q2b * N;
#pragma unroll
          for (int s = 0; s < KS_N; ++s) {
            const int q1 = min(4 * s + lc, N - 1);
            y[t][0][s] = Yb[q1];
            y[t][1][s] = Yb[P * N2 + q1];
            y[t][2][s] = Yb[2 * P * N2 + q1];
          }
        }
        double zb[JPW][2], zg[JPW][2];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          zb[t][0] = zb[t][1] = zg[t][0] = zg[t][1] = 0.0;
#pragma unroll
          for (int s = 0; s < KS_N; ++s) {
            dmma(zb[t][0], zb[t][1], fBt[s], y[t][0][s]);
            dmma(zb[t][0], zb[t][1], fGt[s], y[t][1][s]);
            dmma(zg[t][0], zg[t][1], fBt[s], y[t][2][s]);
          }
        }
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = kwarp + (t0 + t) * NKWW;
          const int c = j / NTL, tl = j - c * NTL;
#pragma unroll
          for (int i = 0; i < 2; ++i) {
            const int n = tl * 8 + 2 * lc + i;
            if (j < NJ && lr < P && n < NC) {
              const int q2 = n / P, a0 = n - q2 * P;
              Wr[Dm::O_Z + ((c * 2 + 0) * N + q2) * P2 + lr * P + a0] = zb[t][i];
              Wr[Dm::O_Z + ((c * 2 + 1) * N + q2) * P2 + lr * P + a0] = zg[t][i];
            }
          }
        }
      }
      constexpr int NCE = N * T, NTE = (NCE + 7) / 8;   // ZE = Phi^T . YE
      for (int te = kwarp; te < NTE; te += NKWW) {
        const int nb = min(te * 8 + lr, NCE - 1);
        const int q2b = nb / T, j0b = nb - q2b * T;
        double d0 = 0.0, d1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_N; ++s) dmma(d0, d1, fPt[s], Wr[Dm::O_YE + j0b * N2 + q2b * N + min(4 * s + lc, N - 1)]);
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = te * 8 + 2 * lc + i;
          if (lr < T && n < NCE) {
            const int q2 = n / T, j0 = n - q2 * T;
            Wr[Dm::O_ZE + q2 * T2 + lr * T + j0] = i ? d1 : d0;
          }
        }
      }
    }
    kw_bar<NKW>();
    kstamp(5);
    {   // A^T -> global F_z.1 (zone-local) and F^T v
      constexpr int NTL = (P2 + 7) / 8, NJ = 3 * NTL, JPWT = (NJ + NKWW - 1) / NKWW, JPW = JPWT < KWCH ? JPWT : KWCH;
      for (int t0 = 0; t0 < JPWT; t0 += JPW) {
        double zv[JPW][2][KS_N];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = min(kwarp + (t0 + t) * NKWW, NJ - 1);
          const int c = j / NTL, tl = j - c * NTL;
          const int nb = min(tl * 8 + lr, P2 - 1);
          const double *Zb = Wr + Dm::O_Z + c * 2 * N * P2 + nb;
#pragma unroll
          for (int s = 0; s < KS_N; ++s) {
            const int q2 = min(4 * s + lc, N - 1);
            zv[t][0][s] = Zb[q2 * P2];
            zv[t][1][s] = Zb[(N + q2) * P2];
          }
        }
        double d[JPW][2];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          d[t][0] = d[t][1] = 0.0;
#pragma unroll
          for (int s = 0; s < KS_N; ++s) {
            dmma(d[t][0], d[t][1], fBt[s], zv[t][0][s]);
            dmma(d[t][0], d[t][1], fGt[s], zv[t][1][s]);
          }
        }
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = kwarp + (t0 + t) * NKWW;
          const int c = j / NTL, tl = j - c * NTL;
          if (j < NJ && lr < P) {
#pragma unroll
            for (int i = 0; i < 2; ++i) {
              const int n = tl * 8 + 2 * lc + i;
              if (n < P2) a.Fz1[(z * 3 + c) * P3 + lr * P2 + n] = d[t][i];
            }
          }
        }
      }
      constexpr int NTE = (T2 + 7) / 8;
      for (int te = kwarp; te < NTE; te += NKWW) {
        const int nb = min(te * 8 + lr, T2 - 1);
        double d0 = 0.0, d1 = 0.0;
#pragma unroll
        for (int s = 0; s < KS_N; ++s) dmma(d0, d1, fPt[s], Wr[Dm::O_ZE + min(4 * s + lc, N - 1) * T2 + nb]);
        if (lr < T) {
#pragma unroll
          for (int i = 0; i < 2; ++i) {
            const int n = te * 8 + 2 * lc + i;
            if (n < T2) a.FTv[z * T3 + lr * T2 + n] = i ? d1 : d0;
          }
        }
      }
    }
    kw_bar<NKW>();   // Y/Z scratch free again (the next forward pass overwrites it)
    kstamp(6);
  };

  // ---------------- PW: stage C (velocity, e) + point evaluation of zone z ----------------
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;
  const int pr = tid, q0a = pr % NH, q1 = (pr / NH) % N, q2 = pr / (NH * N);
  auto pw_point = [&](const double *ub, const double *js, double *jb, int64_t z) {
    // both points of the thread (q0a, q0a + N/2) share every U load; their physics is independent ILP
    const double gamma = js[9];
    const int qa = (q2 * N + q1) * N + q0a, qb = qa + NH;
    const double Ra = ub[Dm::O_R + qa], Rb = ub[Dm::O_R + qb];
    double ga[9], gb[9];
#pragma unroll
    for (int i = 0; i < 9; ++i) { ga[i] = 0.0; gb[i] = 0.0; }
#pragma unroll
    for (int a0 = 0; a0 < P; ++a0) {
      const double ba = tB[q0a * P + a0], gga = tG[q0a * P + a0];
      const double bb = tB[(q0a + NH) * P + a0], ggb = tG[(q0a + NH) * P + a0];
#pragma unroll
      for (int f = 0; f < 3; ++f)
#pragma unroll
        for (int m = 0; m < 3; ++m) {
          const double u = ub[(((f * 3 + m) * N + q2) * N + q1) * P + a0];
          ga[f * 3 + m] = fma(m == 0 ? gga : ba, u, ga[f * 3 + m]);
          gb[f * 3 + m] = fma(m == 0 ? ggb : bb, u, gb[f * 3 + m]);
        }
    }
    double ea = 0.0, eb = 0.0;
#pragma unroll
    for (int j0 = 0; j0 < T; ++j0) {
      const double ue = ub[Dm::O_UE + (q2 * N + q1) * T + j0];
      ea = fma(tPhi[q0a * T + j0], ue, ea);
      eb = fma(tPhi[(q0a + NH) * T + j0], ue, eb);
    }
    double Ja[3][3], Gva[3][3], Jb[3][3], Gvb[3][3];
#pragma unroll
    for (int c = 0; c < 3; ++c)
#pragma unroll
      for (int d = 0; d < 3; ++d) {
        Ja[c][d] = jb[(c * 3 + d) * N3 + qa]; Gva[c][d] = ga[c * 3 + d];
        Jb[c][d] = jb[(c * 3 + d) * N3 + qb]; Gvb[c][d] = gb[c * 3 + d];
      }
    const double w12 = sW[q1] * sW[q2];
    PointOut<3> oa, ob;
    const double best = sRed[8];   // largest exact inverse dt found so far by this CTA (dt filter)
    point_eval3<true>(Ja, Gva, ea, Ra, sW[q0a] * w12, gamma, js, a.ph, oa, best);
    point_eval3<true>(Jb, Gvb, eb, Rb, sW[q0a + NH] * w12, gamma, js, a.ph, ob, best);
    {
      double mi = fmax(oa.inv, ob.inv);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) mi = fmax(mi, __shfl_xor_sync(0xffffffffu, mi, o));
      if ((threadIdx.x & 31) == 0 && mi > best)
        atomicMax(reinterpret_cast<unsigned long long *>(sRed + 8), (unsigned long long)__double_as_longlong(mi));
    }
#pragma unroll
    for (int cd = 0; cd < 9; ++cd) {     // in place over J: only this thread touches slots qa, qb
      jb[cd * N3 + qa] = oa.S[cd / 3][cd % 3];
      jb[cd * N3 + qb] = ob.S[cd / 3][cd % 3];
    }
    jb[Dm::O_PQ + qa] = oa.P;
    jb[Dm::O_PQ + qb] = ob.P;
    if (a.Sq != nullptr) {
#pragma unroll
      for (int cd = 0; cd < 9; ++cd) {
        a.Sq[(z * N3 + qa) * 9 + cd] = oa.S[cd / 3][cd % 3];
        a.Sq[(z * N3 + qb) * 9 + cd] = ob.S[cd / 3][cd % 3];
      }
    }
    dtmin = fmin(dtmin, fmin(oa.dt, ob.dt));
    bad |= oa.bad | ob.bad;
  };

  // ---------------- the two groups run separate code paths from here on (register split) ----------------
  // Both execute the same number of CTA barriers (bar 0): 1 after the prologue + (nz + 1) in the loop.
  if (is_kw) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;\n" ::"n"(Cfg::REG_KW));
    if (a.prof != nullptr && tid == NPW) {
      for (int sl = 0; sl < 16; ++sl) sKP[sl] = 0;
      sKP[15] = clock64();
    }
    kw_load_id(0);
    cp_async_commit();
    cp_async_wait<0>();
    kw_bar<NKW>();                   // ids of zone 0
    kw_issue(0);
    kw_load_id(1);
    cp_async_commit();
    cp_async_wait<0>();
    kw_bar<NKW>();
    if (nz > 0 && DIAG != 1) kw_forward(sUV, sJS, sJ);
    cta_bar_div<Cfg::NTH>();
    long long t_work = 0;
    for (int64_t i = 0; i <= nz; ++i) {
      const long long t0 = clock64();
      kw_issue(i + 1);                 // gather of zone i+1 flies while the back stages of zone i-1 run
      kw_load_id(i + 2);
      cp_async_commit();
      kstamp(3);
      if (i >= 1 && DIAG != 1) kw_back(sJS + ((i - 1) & 1) * Dm::JSBUF, zone_of(i - 1));
      cp_async_wait<0>();
      kw_bar<NKW>();
      kstamp(7);
      if (i + 1 < nz && DIAG != 1)
        kw_forward(sUV + ((i + 1) & 1) * Dm::UVBUF, sJS + ((i + 1) & 1) * Dm::JSBUF, sJ + ((i + 1) & 1) * 10);
      t_work += clock64() - t0;
      cta_bar_div<Cfg::NTH>();
      kstamp(11);
    }
    if (a.prof != nullptr && tid == NPW) {
      a.prof[blockIdx.x * 16 + 1] = t_work;
      for (int sl = 3; sl < 12; ++sl) a.prof[blockIdx.x * 16 + sl] = sKP[sl];
    }
    return;
  }
  asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;\n" ::"n"(Cfg::REG_PW));
  cta_bar_div<Cfg::NTH>();
  long long t_work = 0, t_all = clock64();
  for (int64_t i = 0; i <= nz; ++i) {
    const long long t0 = clock64();
    if (i < nz && tid < TPZ && DIAG != 2)
      pw_point(sUV + (i & 1) * Dm::UVBUF, sJ + (i & 1) * 10, sJS + (i & 1) * Dm::JSBUF, zone_of(i));
    t_work += clock64() - t0;
    cta_bar_div<Cfg::NTH>();
  }
  if (a.prof != nullptr && tid == 0) {
    a.prof[blockIdx.x * 16 + 0] = t_work;
    a.prof[blockIdx.x * 16 + 2] = clock64() - t_all;
  }
  // dt: reduce over the point warps only (named barrier 2), the DMMA warps have exited
  if (bad) dtmin = 0.0;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) dtmin = fmin(dtmin, __shfl_xor_sync(0xffffffffu, dtmin, o));
  if ((tid & 31) == 0) sRed[tid >> 5] = dtmin;
  asm volatile("bar.sync 2, %0;\n" ::"n"(NPW) : "memory");
  if (tid < 32) {
    double r = tid < NPW / 32 ? sRed[tid] : __longlong_as_double(0x7ff0000000000000LL);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) r = fmin(r, __shfl_xor_sync(0xffffffffu, r, o));
    if (tid == 0) a.cta_dt[blockIdx.x] = r;
  }
}
