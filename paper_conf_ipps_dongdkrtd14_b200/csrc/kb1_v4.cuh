// KB1 v4 — warp-specialized, software-pipelined 3D corner force (k <= 4), one persistent CTA per SM.
//
// Same mathematics as kb1_v3.cuh (eq (4)-(6); DESIGN.md §1 rows a0-a5); different schedule.
// The per-stage clock profile of v3 (profiles/) showed every phase latency-bound behind CTA-wide
// barriers: the gather (15%), the DMMA contraction stages (37%) and the point stage (44%) each left the
// FP64 pipe idle while waiting.  v4 splits the CTA into two warp groups that work on DIFFERENT zones:
//
//   PW  (Nq/2 threads, 2 points each): stage C (a0 -> q0, DFMA) + the per-point physics of zone i
//   KW  (4 warps): back stages C^T, B^T, A^T of zone i-1 (DMMA), then the gather (cp.async, issued one
//       zone ahead) and forward stages A, B of zone i+1 (DMMA)
//
// with one CTA barrier per zone and named barriers inside KW.  Double buffers: U (stage B -> C) and
// S (point -> C^T) alternate between zones, so PW and KW never touch the same buffer in an iteration.
// Shared memory (k = 4): U 2 x 6016, S 2 x 5120, KW scratch 5278, tables, J0^{-1}: ~222 KB.
#pragma once
#include "kb1_v3.cuh"

template <int K>
struct V4Dims {
  static constexpr int N = 2 * K, P = K + 1, T = K;
  static constexpr int P2 = P * P, P3 = P * P * P, T2 = T * T, T3 = T * T * T, N2 = N * N, N3 = N * N * N;
  static constexpr int NH = N / 2, TPZ = N3 / 2;
  static constexpr int TAB = (2 * N * P + N * T + N + 1) / 2 * 2;
  // U buffer: U[6][3][N][N][P] UE[N][N][T]
  static constexpr int O_UE = 18 * N2 * P, UBUF = (O_UE + N2 * T + 1) / 2 * 2;
  // S buffer: S[9][N][N][N] Pq[N][N][N]  (layout [cd][q2][q1][q0])
  static constexpr int O_PQ = 9 * N3, SBUF = 10 * N3;
  // KW scratch: XE (X[6][P^3] E[T^3] J0[9] gamma, filled by cp.async) | T/TE aliased with Y/YE + Z/ZE
  static constexpr int XE_X = 0, XE_E = 6 * P3, XE_J = XE_E + T3, XE = (XE_J + 10 + 1) / 2 * 2;
  static constexpr int O_T = 0, O_TE = 12 * N * P2, TREG = O_TE + N * T2;
  static constexpr int O_Y = 0, O_YE = 9 * P * N2, O_Z = O_YE + T * N2, O_ZE = O_Z + 6 * N * P2;
  static constexpr int YZREG = O_ZE + N * T2;
  static constexpr int WREG = (TREG > YZREG ? TREG : YZREG);
  // totals
  static constexpr int OFF_U = TAB, OFF_S = OFF_U + 2 * UBUF, OFF_XE = OFF_S + 2 * SBUF, OFF_W = OFF_XE + XE;
  static constexpr int OFF_J = OFF_W + WREG;            // J0^{-1} + gamma for the two U buffers [2][10]
  static constexpr int OFF_RED = OFF_J + 20;
  static constexpr int TOTAL = OFF_RED + 32;
  static constexpr int MT = (N + 7) / 8, KS_P = (P + 3) / 4, KS_N = (N + 3) / 4, KS_T = (T + 3) / 4;
};

// MODE 0: 2 points per point-thread (Nq/2 threads, 168 registers) + 8 DMMA warps (88 registers)
// MODE 1: 1 point per point-thread (Nq threads, 104 registers)    + 4 DMMA warps (64 registers)
// setmaxnreg only redistributes the CTA's launch allocation (NTH x floor8(65536 / NTH) registers).
template <int K, int MODE>
struct KB1V4Cfg {
  using Dm = V4Dims<K>;
  static constexpr int QPT = MODE == 0 ? 2 : 1;                           // points per point-thread
  static constexpr int NPW = (Dm::N3 / QPT + 127) / 128 * 128;            // whole warpgroups
  static constexpr int NKW = MODE == 0 ? 256 : 128;
  static constexpr int NTH = NPW + NKW;
  // register split by setmaxnreg (the launch gives 65536 / NTH): point warps get more, DMMA warps less
  static constexpr int REG_PW = MODE == 0 ? 168 : 104, REG_KW = MODE == 0 ? 88 : 64;
  static constexpr int KWCH = MODE == 0 ? 8 : 2;                          // DMMA tiles in flight per warp
  static constexpr int REG_LAUNCH = (65536 / NTH) / 8 * 8;
  static_assert(NPW * REG_PW + NKW * REG_KW <= NTH * REG_LAUNCH, "register split exceeds the CTA's allocation");
  static constexpr int SMEM_BYTES = Dm::TOTAL * 8;
};

// thread index read through asm volatile: stops the compiler from hoisting every stage's index arithmetic
// out of the persistent zone loop (which pins registers and spills in the 88-register DMMA warps)
__device__ __forceinline__ int opaque_tid() {
  int t;
  asm volatile("mov.u32 %0, %%tid.x;" : "=r"(t));
  return t;
}

template <int NKW>
__device__ __forceinline__ void kw_bar() { asm volatile("bar.sync 1, %0;\n" ::"n"(NKW) : "memory"); }
// The CTA-wide barrier of the warp-specialized kernels, reached by the point warps and the contraction warps
// at DIFFERENT instructions: the non-aligned barrier.sync with the explicit thread count (legal in divergent
// code; __syncthreads() is barrier.sync.aligned, which requires every thread of the CTA at the same
// instruction — compute-sanitizer synccheck flagged it, gpurun_out r02_sanitizer)
template <int NT>
__device__ __forceinline__ void cta_bar_div() { asm volatile("barrier.sync 0, %0;\n" ::"n"(NT) : "memory"); }

template <int K, int MODE>
__global__ void __launch_bounds__(KB1V4Cfg<K, MODE>::NTH, 1) kb1_v4_3d(const KB1Args a) {
  using Dm = V4Dims<K>;
  using Cfg = KB1V4Cfg<K, MODE>;
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, P2 = Dm::P2, P3 = Dm::P3, T2 = Dm::T2, T3 = Dm::T3;
  constexpr int N2 = Dm::N2, N3 = Dm::N3, NH = Dm::NH, TPZ = Dm::TPZ;
  constexpr int KS_P = Dm::KS_P, KS_N = Dm::KS_N, KS_T = Dm::KS_T;
  constexpr int NPW = Cfg::NPW, NKW = Cfg::NKW, NKWW = NKW / 32, KWCH = Cfg::KWCH;
  static_assert(NKW >= P3, "the gather gives one node per DMMA-warp thread");
  static_assert(Dm::MT == 1, "kb1_v4: rows in one block of 8 (k <= 4)");
  extern __shared__ double smem[];
  double *sTab = smem;
  const double *tB = sTab, *tG = sTab + N * P, *tPhi = sTab + 2 * N * P, *sW = sTab + 2 * N * P + N * T;
  double *sU = smem + Dm::OFF_U, *sS = smem + Dm::OFF_S, *sXE = smem + Dm::OFF_XE, *sWk = smem + Dm::OFF_W;
  double *sJ = smem + Dm::OFF_J, *sRed = smem + Dm::OFF_RED;

  const int tid = threadIdx.x;
  const bool is_kw = tid >= NPW;
  const int ktid = tid - NPW;                       // KW thread index (valid if is_kw)
  const int lane = tid & 31, lr = lane >> 2, lc = lane & 3;
  const int kwarp = ktid >> 5;
  const int64_t Z = a.num_zones, nn = a.num_nodes;
  const int64_t G = gridDim.x;
  const int64_t nz = Z > blockIdx.x ? (Z - 1 - blockIdx.x) / G + 1 : 0;   // zones of this CTA
  auto zone_of = [&](int64_t i) { return (int64_t)blockIdx.x + i * G; };

  for (int i = tid; i < 2 * N * P + N * T + N; i += Cfg::NTH) sTab[i] = __ldg(a.tab + i);
  if (tid == 0) sRed[8] = 0.0;   // dt filter: best exact inverse dt of this CTA (point_eval3<true>)

  // ---------------- KW helpers ----------------
  int32_t nid = -1;   // node id of local node ktid for the next gather (ktid < P3)
  auto kw_load_id = [&](int64_t i) {
    nid = (i < nz && ktid < P3) ? __ldg(a.zone_nodes + zone_of(i) * P3 + ktid) : -1;
  };
  auto kw_issue = [&](int64_t i) {       // cp.async gather of zone i into XE (ids already in nid)
    if (i < nz) {
      const int64_t z = zone_of(i);
      if (ktid < P3) {
        const int64_t node = nid >= 0 ? nid : 0;
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
    }
    cp_async_commit();
  };
  // forward stages A and B of the zone in XE -> U buffer ub (+ J0/gamma -> sJ slot js)
  auto kw_forward = [&](double *ub, double *js) {
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
    double *Tr = sWk;
    {   // stage A: each warp takes tiles kwarp, kwarp + 8, ... of the 6 P^2 columns at once (loads first)
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
      constexpr int NCE = T2, NTE = (NCE + 7) / 8;   // TE = Phi . E (few tiles)
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
    {   // stage B: U0 = B.TB, U1 = G.TB, U2 = B.TG; tiles kwarp, kwarp + 8, ... at once
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
              double *U = ub + (((f * 3) * N + q2) * N + lr) * P + a0;
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
  };
  // back stages C^T, B^T, A^T of zone z from the S buffer sb
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
    {   // B^T: jobs (c, tile) spread over the warps, each warp's jobs loaded/multiplied/stored together
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
    {   // A^T -> global: jobs (c, tile) and the F^T v tiles, each warp's jobs loaded/multiplied/stored together
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
    kw_bar<NKW>();   // Y/Z scratch free again (stage A of the next forward pass overwrites it)
  };

  // ---------------- PW: stage C + point evaluation of zone z from U buffer ub into S buffer sb ----------
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;
  const int pr = tid, q0a = pr % NH, q1 = (pr / NH) % N, q2 = pr / (NH * N);
  auto pw_point = [&](const double *ub, const double *js, double *sb, int64_t z) {
    // both points of the thread (q0a, q0a + N/2) share every U load; their physics is independent ILP
    const double gamma = js[9];
    const int qa = (q2 * N + q1) * N + q0a, qb = qa + NH;
    const double Ra = __ldg(a.rho0detJ0 + z * N3 + qa), Rb = __ldg(a.rho0detJ0 + z * N3 + qb);
    double ga[18], gb[18];
#pragma unroll
    for (int i = 0; i < 18; ++i) { ga[i] = 0.0; gb[i] = 0.0; }
#pragma unroll
    for (int a0 = 0; a0 < P; ++a0) {
      const double ba = tB[q0a * P + a0], gga = tG[q0a * P + a0];
      const double bb = tB[(q0a + NH) * P + a0], ggb = tG[(q0a + NH) * P + a0];
#pragma unroll
      for (int f = 0; f < 6; ++f)
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
        Ja[c][d] = ga[c * 3 + d]; Gva[c][d] = ga[9 + c * 3 + d];
        Jb[c][d] = gb[c * 3 + d]; Gvb[c][d] = gb[9 + c * 3 + d];
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
    for (int cd = 0; cd < 9; ++cd) {
      sb[cd * N3 + qa] = oa.S[cd / 3][cd % 3];
      sb[cd * N3 + qb] = ob.S[cd / 3][cd % 3];
    }
    sb[Dm::O_PQ + qa] = oa.P;
    sb[Dm::O_PQ + qb] = ob.P;
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

  auto pw_point1 = [&](const double *ub, const double *js, double *sb, int64_t z) {
    // one point per thread: q = tid
    const int q0 = tid % N, q1s = (tid / N) % N, q2s = tid / N2;
    const int q = tid;
    const double R = __ldg(a.rho0detJ0 + z * N3 + q);
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
          g[f * 3 + m] = fma(m == 0 ? gg : b, ub[(((f * 3 + m) * N + q2s) * N + q1s) * P + a0], g[f * 3 + m]);
    }
    double eq = 0.0;
#pragma unroll
    for (int j0 = 0; j0 < T; ++j0) eq = fma(tPhi[q0 * T + j0], ub[Dm::O_UE + (q2s * N + q1s) * T + j0], eq);
    double Jm[3][3], Gv[3][3];
#pragma unroll
    for (int c = 0; c < 3; ++c)
#pragma unroll
      for (int d = 0; d < 3; ++d) { Jm[c][d] = g[c * 3 + d]; Gv[c][d] = g[9 + c * 3 + d]; }
    PointOut<3> o;
    point_eval3(Jm, Gv, eq, R, sW[q0] * sW[q1s] * sW[q2s], js[9], js, a.ph, o);
#pragma unroll
    for (int cd = 0; cd < 9; ++cd) sb[cd * N3 + q] = o.S[cd / 3][cd % 3];
    sb[Dm::O_PQ + q] = o.P;
    if (a.Sq != nullptr) {
#pragma unroll
      for (int cd = 0; cd < 9; ++cd) a.Sq[(z * N3 + q) * 9 + cd] = o.S[cd / 3][cd % 3];
    }
    dtmin = fmin(dtmin, o.dt);
    bad |= o.bad;
  };

  // ---------------- the two groups run separate code paths from here on (register split) ----------------
  // Both execute the same number of CTA barriers (bar 0): 1 after the prologue + (nz + 1) in the loop.
  if (is_kw) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;\n" ::"n"(Cfg::REG_KW));
    kw_load_id(0);
    kw_issue(0);
    kw_load_id(1);
    cp_async_wait<0>();
    kw_bar<NKW>();
    if (nz > 0) kw_forward(sU, sJ);
    __syncthreads();
    long long t_work = 0;
    for (int64_t i = 0; i <= nz; ++i) {
      const long long t0 = clock64();
      kw_issue(i + 1);                 // gather of zone i+1 flies while the back stages of zone i-1 run
      kw_load_id(i + 2);
      if (i >= 1) kw_back(sS + ((i - 1) & 1) * Dm::SBUF, zone_of(i - 1));
      cp_async_wait<0>();
      kw_bar<NKW>();
      if (i + 1 < nz) kw_forward(sU + ((i + 1) & 1) * Dm::UBUF, sJ + ((i + 1) & 1) * 10);
      t_work += clock64() - t0;
      __syncthreads();
    }
    if (a.prof != nullptr && tid == NPW) a.prof[blockIdx.x * 16 + 1] = t_work;
    return;
  }
  asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;\n" ::"n"(Cfg::REG_PW));
  __syncthreads();
  long long t_work = 0, t_all = clock64();
  for (int64_t i = 0; i <= nz; ++i) {
    const long long t0 = clock64();
    if (MODE == 0) {
      if (i < nz && tid < TPZ) pw_point(sU + (i & 1) * Dm::UBUF, sJ + (i & 1) * 10, sS + (i & 1) * Dm::SBUF, zone_of(i));
    } else {
      if (i < nz && tid < N3) pw_point1(sU + (i & 1) * Dm::UBUF, sJ + (i & 1) * 10, sS + (i & 1) * Dm::SBUF, zone_of(i));
    }
    t_work += clock64() - t0;
    __syncthreads();
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
