// KB1 — fused zone-batch corner-force kernel for sm_100a (FP64, CUDA cores).
//
// One CTA owns ZPC zones.  It replaces the paper's kernels 1-8 and 10 (Table 2):
//   a0 gather   X_z, V_z through the zone->node map, E_z, J0^{-1}_z into shared memory
//   a1/a2       J(q) = X_z grad W(q), grad^v(q) = V_z grad W(q), e(q) = E_z phi(q) by sum factorization
//               with the 1-D GLL-Lagrange / Bernstein tables (kernel 3)
//   a2/a3       per-point geometry, EOS, viscosity, stress, dt in registers (kernels 1, 2, 5, 6)
//   a4/a5       back contractions without forming A_z or F_z (kernels 4, 7, 8, 10):
//                 (F_z 1)_{c,a} = sum_q sum_d S_cd(q) dW_a/dxi_d(q)   [= A_z (B^T 1), B^T 1 = 1]
//                 (F_z^T V)_j   = sum_q phi_j(q) (S(q) : grad^v(q))    [= B (A_z^T V)]
//               F_z.1 goes to a zone-local buffer (gathered deterministically by KB2), F_z^T v straight
//               to out_FTv, and the CTA's min dt to a per-CTA slot.
//
// 3D: thread (q0, q1) of a zone, looping over q2 slabs; 2D: thread per point, one pass.
#pragma once
#include "pointwise.cuh"

struct KB1Args {
  const double *x, *v, *e, *rho0detJ0;
  const int32_t *zone_nodes;
  const double *J0inv;     // [Z][D*D] per zone (affine initial zones)
  const double *J0inv_q;   // [Z][NQ][D*D] per point (non-affine initial zones, read by the v1 kernels only), else nullptr
  const double *zone_gamma;// [Z]
  const double *tab;       // [B: N*P][G: N*P][Phi: N*T][w: N]
  double *Fz1;             // [Z][D][NK] zone-local F_z.1
  double *FTv;             // [Z][NT]
  double *cta_dt;          // [gridDim.x]
  double *Sq;              // debug only (tests): S(q) = alpha sigma adj(J)^T as [Z][NQ][D*D], else nullptr
  long long *prof;         // debug only: per-CTA clock64 stamps at the stage barriers [grid][16], else nullptr
  int64_t num_zones, num_nodes;
  CFPhys ph;
  int32_t zero;            // always 0 (an offset the compiler cannot fold: kb1_v6.cuh)
};

__device__ __forceinline__ double block_min(double v, double *red) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmin(v, __shfl_xor_sync(0xffffffffu, v, o));
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (lane == 0) red[w] = v;
  __syncthreads();
  if (w == 0) {
    const int nw = (blockDim.x + 31) >> 5;
    double r = lane < nw ? red[lane] : __longlong_as_double(0x7ff0000000000000LL);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) r = fmin(r, __shfl_xor_sync(0xffffffffu, r, o));
    v = r;
  }
  return v;
}

template <int K>
struct Dims3 {
  static constexpr int D = 3, N = 2 * K, P = K + 1, T = K;
  static constexpr int NK = P * P * P, NT = T * T * T, NQ = N * N * N, NS = N * N, NF = 6;
  // per-zone shared-memory regions (doubles)
  static constexpr int SZ_X = NF * NK, SZ_E = NT, SZ_ACCF = D * NK, SZ_ACCE = NT, SZ_J0 = 9;
  static constexpr int SZ_S = 9 * NS, SZ_P = NS;
  static constexpr int SZ_T_FWD = 2 * NF * P * P + T * T;          // TB, TG, TE
  static constexpr int SZ_T_BCK = 9 * N * P + N * T;               // Y, YE
  static constexpr int SZ_T = SZ_T_FWD > SZ_T_BCK ? SZ_T_FWD : SZ_T_BCK;
  static constexpr int SZ_U_FWD = 3 * NF * N * P + N * T;          // U, UE
  static constexpr int SZ_U_BCK = 2 * D * P * P + T * T;           // ZB/ZG, ZE
  static constexpr int SZ_U = SZ_U_FWD > SZ_U_BCK ? SZ_U_FWD : SZ_U_BCK;
  // two reused regions per zone:  A = T/TE -> S/Pq -> Z/ZE,  B = U/UE -> Y/YE
  static constexpr int SZ_A0 = SZ_T_FWD > SZ_S + SZ_P ? SZ_T_FWD : SZ_S + SZ_P;
  static constexpr int SZ_A = SZ_A0 > SZ_U_BCK ? SZ_A0 : SZ_U_BCK;
  static constexpr int SZ_B = SZ_U_FWD > SZ_T_BCK ? SZ_U_FWD : SZ_T_BCK;
  static constexpr int ZONE = SZ_X + SZ_E + SZ_ACCF + SZ_ACCE + SZ_J0 + SZ_A + SZ_B;
  static constexpr int TAB = 2 * N * P + N * T + N;
};

template <int K, int ZPC>
struct KB1Cfg3 {
  using Dm = Dims3<K>;
  static constexpr int NTH = (ZPC * Dm::NS + 31) / 32 * 32;   // padded to whole warps
  static constexpr int SMEM_DOUBLES = Dm::TAB + ZPC * Dm::ZONE + 32;
  static constexpr int SMEM_BYTES = SMEM_DOUBLES * 8;
};

template <int K, int ZPC, int MINB>
__global__ void __launch_bounds__(KB1Cfg3<K, ZPC>::NTH, MINB) kb1_corner_force_3d(const KB1Args a) {
  using Dm = Dims3<K>;
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, NK = Dm::NK, NT = Dm::NT, NS = Dm::NS, NF = Dm::NF;
  constexpr int NTH = KB1Cfg3<K, ZPC>::NTH;
  constexpr int P2 = P * P, T2 = T * T;
  extern __shared__ double smem[];
  double *sB = smem, *sG = sB + N * P, *sPhi = sG + N * P, *sW = sPhi + N * T;
  double *zb = smem + Dm::TAB;
  double *sX = zb;                                // [ZPC][NF][NK]
  double *sE = sX + ZPC * Dm::SZ_X;               // [ZPC][NT]
  double *sAF = sE + ZPC * Dm::SZ_E;              // [ZPC][3][NK]
  double *sAE = sAF + ZPC * Dm::SZ_ACCF;          // [ZPC][NT]
  double *sJ0 = sAE + ZPC * Dm::SZ_ACCE;          // [ZPC][9]
  double *sRA = sJ0 + ZPC * Dm::SZ_J0;             // [ZPC][SZ_A]  TB/TG/TE | S[9][NS] Pq[NS] | ZB/ZG/ZE
  double *sRB = sRA + ZPC * Dm::SZ_A;               // [ZPC][SZ_B]  U/UE     | Y/YE
  double *sRed = sRB + ZPC * Dm::SZ_B;             // [32]

  const int tid = threadIdx.x;
  const int64_t zone0 = (int64_t)blockIdx.x * ZPC;
  const int64_t Z = a.num_zones, nn = a.num_nodes;

  // ---- a0: tables + gather --------------------------------------------------------------------
  for (int i = tid; i < Dm::TAB; i += NTH) smem[i] = a.tab[i];
  for (int i = tid; i < ZPC * NK; i += NTH) {
    const int zl = i / NK, r = i - zl * NK;
    const int64_t z = zone0 + zl;
    double vals[6] = {0, 0, 0, 0, 0, 0};
    if (z < Z) {
      const int64_t node = a.zone_nodes[z * NK + r];
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        vals[c] = __ldg(a.x + c * nn + node);
        vals[3 + c] = __ldg(a.v + c * nn + node);
      }
    }
#pragma unroll
    for (int f = 0; f < 6; ++f) sX[(zl * NF + f) * NK + r] = vals[f];
#pragma unroll
    for (int c = 0; c < 3; ++c) sAF[(zl * 3 + c) * NK + r] = 0.0;
  }
  for (int i = tid; i < ZPC * NT; i += NTH) {
    const int zl = i / NT, r = i - zl * NT;
    const int64_t z = zone0 + zl;
    sE[i] = (z < Z) ? __ldg(a.e + z * NT + r) : 0.0;
    sAE[i] = 0.0;
  }
  for (int i = tid; i < ZPC * 9; i += NTH) {
    const int zl = i / 9, r = i - zl * 9;
    const int64_t z = zone0 + zl;
    sJ0[i] = (z < Z) ? __ldg(a.J0inv + z * 9 + r) : (r % 4 == 0 ? 1.0 : 0.0);
  }
  __syncthreads();

  // ---- per-thread identity ----------------------------------------------------------------------
  const int my_zl = tid / NS, my_qq = tid - my_zl * NS;
  const int q0 = my_qq % N, q1 = my_qq / N;
  const bool has_point = my_zl < ZPC;            // padding threads only help with the contractions
  const int64_t my_z = zone0 + my_zl;
  const bool active = has_point && my_z < Z;
  const double gamma = active ? __ldg(a.zone_gamma + my_z) : 1.4;
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;

  for (int q2 = 0; q2 < N; ++q2) {
    // ---- stage A: contract a2 -> q2 (values and derivatives), e: j2 -> q2 ------------------------
    for (int i = tid; i < ZPC * NF * P2; i += NTH) {
      const int zl = i / (NF * P2), rr = i - zl * (NF * P2);
      const int f = rr / P2, r = rr - f * P2;
      const double *X = sX + (zl * NF + f) * NK + r;
      double tb = 0.0, tg = 0.0;
#pragma unroll
      for (int a2 = 0; a2 < P; ++a2) {
        const double xv = X[a2 * P2];
        tb = fma(sB[q2 * P + a2], xv, tb);
        tg = fma(sG[q2 * P + a2], xv, tg);
      }
      double *Tz = sRA + zl * Dm::SZ_A;
      Tz[f * P2 + r] = tb;
      Tz[NF * P2 + f * P2 + r] = tg;
    }
    for (int i = tid; i < ZPC * T2; i += NTH) {
      const int zl = i / T2, r = i - zl * T2;
      const double *Ez = sE + zl * NT + r;
      double te = 0.0;
#pragma unroll
      for (int j2 = 0; j2 < T; ++j2) te = fma(sPhi[q2 * T + j2], Ez[j2 * T2], te);
      sRA[zl * Dm::SZ_A + 2 * NF * P2 + r] = te;
    }
    __syncthreads();
    // ---- stage B: contract a1 -> q1 --------------------------------------------------------------
    for (int i = tid; i < ZPC * NF * N * P; i += NTH) {
      const int zl = i / (NF * N * P), rr = i - zl * (NF * N * P);
      const int f = rr / (N * P), r2 = rr - f * (N * P);
      const int qq1 = r2 / P, a0 = r2 - qq1 * P;
      const double *Tz = sRA + zl * Dm::SZ_A;
      const double *TB = Tz + f * P2 + a0, *TG = Tz + NF * P2 + f * P2 + a0;
      double u0 = 0.0, u1 = 0.0, u2 = 0.0;
#pragma unroll
      for (int a1 = 0; a1 < P; ++a1) {
        const double b = sB[qq1 * P + a1], g = sG[qq1 * P + a1];
        const double tb = TB[a1 * P], tg = TG[a1 * P];
        u0 = fma(b, tb, u0);
        u1 = fma(g, tb, u1);
        u2 = fma(b, tg, u2);
      }
      double *Uz = sRB + zl * Dm::SZ_B + f * 3 * N * P;
      Uz[0 * N * P + r2] = u0;
      Uz[1 * N * P + r2] = u1;
      Uz[2 * N * P + r2] = u2;
    }
    for (int i = tid; i < ZPC * N * T; i += NTH) {
      const int zl = i / (N * T), r = i - zl * (N * T);
      const int qq1 = r / T, j0 = r - qq1 * T;
      const double *TE = sRA + zl * Dm::SZ_A + 2 * NF * P2 + j0;
      double ue = 0.0;
#pragma unroll
      for (int j1 = 0; j1 < T; ++j1) ue = fma(sPhi[qq1 * T + j1], TE[j1 * T], ue);
      sRB[zl * Dm::SZ_B + 3 * NF * N * P + r] = ue;
    }
    __syncthreads();
    // ---- stage C + point evaluation --------------------------------------------------------------
    if (has_point) {
      const double *Uz = sRB + my_zl * Dm::SZ_B;
      double Jm[3][3], Gv[3][3];
#pragma unroll
      for (int f = 0; f < NF; ++f) {
        const double *U = Uz + f * 3 * N * P + q1 * P;
        double d0 = 0.0, d1 = 0.0, d2 = 0.0;
#pragma unroll
        for (int a0 = 0; a0 < P; ++a0) {
          const double b = sB[q0 * P + a0], g = sG[q0 * P + a0];
          d0 = fma(g, U[a0], d0);
          d1 = fma(b, U[N * P + a0], d1);
          d2 = fma(b, U[2 * N * P + a0], d2);
        }
        if (f < 3) { Jm[f][0] = d0; Jm[f][1] = d1; Jm[f][2] = d2; }
        else { Gv[f - 3][0] = d0; Gv[f - 3][1] = d1; Gv[f - 3][2] = d2; }
      }
      const double *UE = Uz + 3 * NF * N * P + q1 * T;
      double eq = 0.0;
#pragma unroll
      for (int j0 = 0; j0 < T; ++j0) eq = fma(sPhi[q0 * T + j0], UE[j0], eq);
      const int q = (q2 * N + q1) * N + q0;
      const double R = active ? __ldg(a.rho0detJ0 + my_z * Dm::NQ + q) : 1.0;
      const double alpha = sW[q0] * sW[q1] * sW[q2];
      PointOut<3> o;
      const double *j0p = (a.J0inv_q != nullptr && active) ? a.J0inv_q + (my_z * Dm::NQ + q) * 9 : sJ0 + my_zl * 9;
      point_eval3(Jm, Gv, eq, R, alpha, gamma, j0p, a.ph, o);
      double *S = sRA + my_zl * Dm::SZ_A + my_qq;
#pragma unroll
      for (int c = 0; c < 3; ++c)
#pragma unroll
        for (int d = 0; d < 3; ++d) S[(c * 3 + d) * NS] = o.S[c][d];
      sRA[my_zl * Dm::SZ_A + Dm::SZ_S + my_qq] = o.P;
      if (a.Sq != nullptr && active) {
#pragma unroll
        for (int c = 0; c < 9; ++c) a.Sq[(my_z * Dm::NQ + q) * 9 + c] = o.S[c / 3][c % 3];
      }
      if (active) {
        dtmin = fmin(dtmin, o.dt);
        bad |= o.bad;
      }
    }
    __syncthreads();
    // ---- stage C^T: contract q0 -> a0 -------------------------------------------------------------
    for (int i = tid; i < ZPC * 3 * N * P; i += NTH) {
      const int zl = i / (3 * N * P), rr = i - zl * (3 * N * P);
      const int c = rr / (N * P), r2 = rr - c * (N * P);
      const int qq1 = r2 / P, a0 = r2 - qq1 * P;
      const double *S = sRA + zl * Dm::SZ_A + qq1 * N;
      double y0 = 0.0, y1 = 0.0, y2 = 0.0;
#pragma unroll
      for (int qq0 = 0; qq0 < N; ++qq0) {
        const double b = sB[qq0 * P + a0], g = sG[qq0 * P + a0];
        y0 = fma(g, S[(c * 3 + 0) * NS + qq0], y0);
        y1 = fma(b, S[(c * 3 + 1) * NS + qq0], y1);
        y2 = fma(b, S[(c * 3 + 2) * NS + qq0], y2);
      }
      double *Y = sRB + zl * Dm::SZ_B + c * 3 * N * P;
      Y[0 * N * P + r2] = y0;
      Y[1 * N * P + r2] = y1;
      Y[2 * N * P + r2] = y2;
    }
    for (int i = tid; i < ZPC * N * T; i += NTH) {
      const int zl = i / (N * T), r = i - zl * (N * T);
      const int qq1 = r / T, j0 = r - qq1 * T;
      const double *Pz = sRA + zl * Dm::SZ_A + Dm::SZ_S + qq1 * N;
      double ye = 0.0;
#pragma unroll
      for (int qq0 = 0; qq0 < N; ++qq0) ye = fma(sPhi[qq0 * T + j0], Pz[qq0], ye);
      sRB[zl * Dm::SZ_B + 9 * N * P + r] = ye;
    }
    __syncthreads();
    // ---- stage B^T: contract q1 -> a1 -------------------------------------------------------------
    for (int i = tid; i < ZPC * 3 * P2; i += NTH) {
      const int zl = i / (3 * P2), rr = i - zl * (3 * P2);
      const int c = rr / P2, r = rr - c * P2;
      const int a1 = r / P, a0 = r - a1 * P;
      const double *Y = sRB + zl * Dm::SZ_B + c * 3 * N * P + a0;
      double zbv = 0.0, zgv = 0.0;
#pragma unroll
      for (int qq1 = 0; qq1 < N; ++qq1) {
        const double b = sB[qq1 * P + a1], g = sG[qq1 * P + a1];
        zbv = fma(b, Y[qq1 * P], zbv);
        zbv = fma(g, Y[N * P + qq1 * P], zbv);
        zgv = fma(b, Y[2 * N * P + qq1 * P], zgv);
      }
      double *Zr = sRA + zl * Dm::SZ_A;
      Zr[c * P2 + r] = zbv;
      Zr[3 * P2 + c * P2 + r] = zgv;
    }
    for (int i = tid; i < ZPC * T2; i += NTH) {
      const int zl = i / T2, r = i - zl * T2;
      const int j1 = r / T, j0 = r - j1 * T;
      const double *YE = sRB + zl * Dm::SZ_B + 9 * N * P + j0;
      double ze = 0.0;
#pragma unroll
      for (int qq1 = 0; qq1 < N; ++qq1) ze = fma(sPhi[qq1 * T + j1], YE[qq1 * T], ze);
      sRA[zl * Dm::SZ_A + 6 * P2 + r] = ze;
    }
    __syncthreads();
    // ---- stage A^T: accumulate q2 -> a2 -----------------------------------------------------------
    for (int i = tid; i < ZPC * 3 * NK; i += NTH) {
      const int zl = i / (3 * NK), rr = i - zl * (3 * NK);
      const int c = rr / NK, r3 = rr - c * NK;
      const int a2 = r3 / P2, r = r3 - a2 * P2;
      const double *Zr = sRA + zl * Dm::SZ_A;
      sAF[i] = fma(sB[q2 * P + a2], Zr[c * P2 + r], fma(sG[q2 * P + a2], Zr[3 * P2 + c * P2 + r], sAF[i]));
    }
    for (int i = tid; i < ZPC * NT; i += NTH) {
      const int zl = i / NT, r3 = i - zl * NT;
      const int j2 = r3 / T2, r = r3 - j2 * T2;
      sAE[i] = fma(sPhi[q2 * T + j2], sRA[zl * Dm::SZ_A + 6 * P2 + r], sAE[i]);
    }
    __syncthreads();   // region A (Z read above) is overwritten by the next slab's stage A
  }
  __syncthreads();
  // ---- outputs ----------------------------------------------------------------------------------
  for (int i = tid; i < ZPC * 3 * NK; i += NTH) {
    const int zl = i / (3 * NK);
    if (zone0 + zl < Z) a.Fz1[zone0 * 3 * NK + i] = sAF[i];
  }
  for (int i = tid; i < ZPC * NT; i += NTH) {
    const int zl = i / NT;
    if (zone0 + zl < Z) a.FTv[zone0 * NT + i] = sAE[i];
  }
  if (bad) dtmin = 0.0;
  const double m = block_min(dtmin, sRed);
  if (tid == 0) a.cta_dt[blockIdx.x] = m;
}

// =================================================================================================
// 2D: one thread per quadrature point, all contractions in one pass
// =================================================================================================
template <int K>
struct Dims2 {
  static constexpr int D = 2, N = 2 * K, P = K + 1, T = K;
  static constexpr int NK = P * P, NT = T * T, NQ = N * N, NF = 4;
  static constexpr int SZ_X = NF * NK, SZ_E = NT;
  static constexpr int SZ_T = 2 * NF * N * P + N * T;   // TB[f][q1][a0], TG[f][q1][a0], TE[q1][j0]
  static constexpr int SZ_S = 4 * NQ + NQ;              // S[4][NQ], P[NQ]
  static constexpr int SZ_Y = 2 * 2 * N * P + N * T;    // Y[c][2][q1][a0], YE[q1][j0]
  static constexpr int ZONE = SZ_X + SZ_E + 4 + SZ_T + SZ_S + SZ_Y;
  static constexpr int TAB = 2 * N * P + N * T + N;
};

template <int K, int ZPC>
struct KB1Cfg2 {
  using Dm = Dims2<K>;
  static constexpr int NTH = (ZPC * Dm::NQ + 31) / 32 * 32;   // padded to whole warps
  static constexpr int SMEM_DOUBLES = Dm::TAB + ZPC * Dm::ZONE + 32;
  static constexpr int SMEM_BYTES = SMEM_DOUBLES * 8;
};

template <int K, int ZPC, int MINB>
__global__ void __launch_bounds__(KB1Cfg2<K, ZPC>::NTH, MINB) kb1_corner_force_2d(const KB1Args a) {
  using Dm = Dims2<K>;
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, NK = Dm::NK, NT = Dm::NT, NQ = Dm::NQ, NF = Dm::NF;
  constexpr int NTH = KB1Cfg2<K, ZPC>::NTH;
  extern __shared__ double smem[];
  double *sB = smem, *sG = sB + N * P, *sPhi = sG + N * P, *sW = sPhi + N * T;
  double *zb = smem + Dm::TAB;
  double *sX = zb;                          // [ZPC][NF][NK]
  double *sE = sX + ZPC * Dm::SZ_X;         // [ZPC][NT]
  double *sJ0 = sE + ZPC * Dm::SZ_E;        // [ZPC][4]
  double *sT = sJ0 + ZPC * 4;               // [ZPC][SZ_T]
  double *sS = sT + ZPC * Dm::SZ_T;         // [ZPC][SZ_S]
  double *sY = sS + ZPC * Dm::SZ_S;         // [ZPC][SZ_Y]
  double *sRed = sY + ZPC * Dm::SZ_Y;

  const int tid = threadIdx.x;
  const int64_t zone0 = (int64_t)blockIdx.x * ZPC;
  const int64_t Z = a.num_zones, nn = a.num_nodes;

  for (int i = tid; i < Dm::TAB; i += NTH) smem[i] = a.tab[i];
  // the point stage's global operands (rho0|J0| of this thread's point, gamma of its zone) are loaded
  // here, so their DRAM latency overlaps the gather instead of stalling the point stage
  const int my_zl = tid / NQ, my_q = tid - my_zl * NQ;
  const bool has_point = my_zl < ZPC;
  const int64_t my_z = zone0 + my_zl;
  const bool active = has_point && my_z < Z;
  const double Rq = active ? __ldg(a.rho0detJ0 + my_z * NQ + my_q) : 1.0;
  const double gamma_z = active ? __ldg(a.zone_gamma + my_z) : 1.4;
  for (int i = tid; i < ZPC * NK; i += NTH) {
    const int zl = i / NK, r = i - zl * NK;
    const int64_t z = zone0 + zl;
    double vals[4] = {0, 0, 0, 0};
    if (z < Z) {
      const int64_t node = a.zone_nodes[z * NK + r];
#pragma unroll
      for (int c = 0; c < 2; ++c) {
        vals[c] = __ldg(a.x + c * nn + node);
        vals[2 + c] = __ldg(a.v + c * nn + node);
      }
    }
#pragma unroll
    for (int f = 0; f < 4; ++f) sX[(zl * NF + f) * NK + r] = vals[f];
  }
  for (int i = tid; i < ZPC * NT; i += NTH) {
    const int zl = i / NT, r = i - zl * NT;
    const int64_t z = zone0 + zl;
    sE[i] = (z < Z) ? __ldg(a.e + z * NT + r) : 0.0;
  }
  for (int i = tid; i < ZPC * 4; i += NTH) {
    const int zl = i / 4, r = i - zl * 4;
    const int64_t z = zone0 + zl;
    sJ0[i] = (z < Z) ? __ldg(a.J0inv + z * 4 + r) : (r % 3 == 0 ? 1.0 : 0.0);
  }
  __syncthreads();
  // stage A: contract a1 -> q1 for every q1: TB[f][q1][a0] = sum_a1 B(q1,a1) X[f][a1][a0] (TG with G)
  for (int i = tid; i < ZPC * NF * N * P; i += NTH) {
    const int zl = i / (NF * N * P), rr = i - zl * (NF * N * P);
    const int f = rr / (N * P), r2 = rr - f * (N * P);
    const int qq1 = r2 / P, a0 = r2 - qq1 * P;
    const double *X = sX + (zl * NF + f) * NK + a0;
    double tb = 0.0, tg = 0.0;
#pragma unroll
    for (int a1 = 0; a1 < P; ++a1) {
      tb = fma(sB[qq1 * P + a1], X[a1 * P], tb);
      tg = fma(sG[qq1 * P + a1], X[a1 * P], tg);
    }
    double *Tz = sT + zl * Dm::SZ_T;
    Tz[f * N * P + r2] = tb;
    Tz[NF * N * P + f * N * P + r2] = tg;
  }
  for (int i = tid; i < ZPC * N * T; i += NTH) {
    const int zl = i / (N * T), r = i - zl * (N * T);
    const int qq1 = r / T, j0 = r - qq1 * T;
    double te = 0.0;
#pragma unroll
    for (int j1 = 0; j1 < T; ++j1) te = fma(sPhi[qq1 * T + j1], sE[zl * NT + j1 * T + j0], te);
    sT[zl * Dm::SZ_T + 2 * NF * N * P + r] = te;
  }
  __syncthreads();
  const int q0 = my_q % N, q1 = my_q / N;
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;
  if (has_point) {
    const double *Tz = sT + my_zl * Dm::SZ_T;
    double Jm[2][2], Gv[2][2];
#pragma unroll
    for (int f = 0; f < NF; ++f) {
      const double *TB = Tz + f * N * P + q1 * P, *TG = Tz + NF * N * P + f * N * P + q1 * P;
      double d0 = 0.0, d1 = 0.0;
#pragma unroll
      for (int a0 = 0; a0 < P; ++a0) {
        d0 = fma(sG[q0 * P + a0], TB[a0], d0);
        d1 = fma(sB[q0 * P + a0], TG[a0], d1);
      }
      if (f < 2) { Jm[f][0] = d0; Jm[f][1] = d1; }
      else { Gv[f - 2][0] = d0; Gv[f - 2][1] = d1; }
    }
    double eq = 0.0;
#pragma unroll
    for (int j0 = 0; j0 < T; ++j0) eq = fma(sPhi[q0 * T + j0], Tz[2 * NF * N * P + q1 * T + j0], eq);
    const double alpha = sW[q0] * sW[q1];
    PointOut<2> o;
    const double *j0p = (a.J0inv_q != nullptr && active) ? a.J0inv_q + (my_z * NQ + my_q) * 4 : sJ0 + my_zl * 4;
    point_eval2(Jm, Gv, eq, Rq, alpha, gamma_z, j0p, a.ph, o);
    double *S = sS + my_zl * Dm::SZ_S;
#pragma unroll
    for (int c = 0; c < 2; ++c)
#pragma unroll
      for (int d = 0; d < 2; ++d) S[(c * 2 + d) * NQ + my_q] = o.S[c][d];
    S[4 * NQ + my_q] = o.P;
    if (a.Sq != nullptr && active) {
#pragma unroll
      for (int c = 0; c < 4; ++c) a.Sq[(my_z * NQ + my_q) * 4 + c] = o.S[c / 2][c % 2];
    }
    if (active) { dtmin = o.dt; bad = o.bad; }
  }
  __syncthreads();
  // C^T: Y[c][0][q1][a0] = sum_q0 G(q0,a0) S_c0 ; Y[c][1][q1][a0] = sum_q0 B(q0,a0) S_c1
  for (int i = tid; i < ZPC * 2 * N * P; i += NTH) {
    const int zl = i / (2 * N * P), rr = i - zl * (2 * N * P);
    const int c = rr / (N * P), r2 = rr - c * (N * P);
    const int qq1 = r2 / P, a0 = r2 - qq1 * P;
    const double *S = sS + zl * Dm::SZ_S + qq1 * N;
    double y0 = 0.0, y1 = 0.0;
#pragma unroll
    for (int qq0 = 0; qq0 < N; ++qq0) {
      y0 = fma(sG[qq0 * P + a0], S[(c * 2 + 0) * NQ + qq0], y0);
      y1 = fma(sB[qq0 * P + a0], S[(c * 2 + 1) * NQ + qq0], y1);
    }
    double *Y = sY + zl * Dm::SZ_Y + c * 2 * N * P;
    Y[r2] = y0;
    Y[N * P + r2] = y1;
  }
  for (int i = tid; i < ZPC * N * T; i += NTH) {
    const int zl = i / (N * T), r = i - zl * (N * T);
    const int qq1 = r / T, j0 = r - qq1 * T;
    const double *Pz = sS + zl * Dm::SZ_S + 4 * NQ + qq1 * N;
    double ye = 0.0;
#pragma unroll
    for (int qq0 = 0; qq0 < N; ++qq0) ye = fma(sPhi[qq0 * T + j0], Pz[qq0], ye);
    sY[zl * Dm::SZ_Y + 4 * N * P + r] = ye;
  }
  __syncthreads();
  // A^T: (F_z 1)[c][a1][a0] = sum_q1 B(q1,a1) Y[c][0][q1][a0] + G(q1,a1) Y[c][1][q1][a0]
  for (int i = tid; i < ZPC * 2 * NK; i += NTH) {
    const int zl = i / (2 * NK), rr = i - zl * (2 * NK);
    const int c = rr / NK, r = rr - c * NK;
    const int a1 = r / P, a0 = r - a1 * P;
    const double *Y = sY + zl * Dm::SZ_Y + c * 2 * N * P + a0;
    double s = 0.0;
#pragma unroll
    for (int qq1 = 0; qq1 < N; ++qq1) {
      s = fma(sB[qq1 * P + a1], Y[qq1 * P], s);
      s = fma(sG[qq1 * P + a1], Y[N * P + qq1 * P], s);
    }
    if (zone0 + zl < Z) a.Fz1[zone0 * 2 * NK + i] = s;
  }
  for (int i = tid; i < ZPC * NT; i += NTH) {
    const int zl = i / NT, r = i - zl * NT;
    const int j1 = r / T, j0 = r - j1 * T;
    const double *YE = sY + zl * Dm::SZ_Y + 4 * N * P + j0;
    double s = 0.0;
#pragma unroll
    for (int qq1 = 0; qq1 < N; ++qq1) s = fma(sPhi[qq1 * T + j1], YE[qq1 * T], s);
    if (zone0 + zl < Z) a.FTv[zone0 * NT + i] = s;
  }
  if (bad) dtmin = 0.0;
  const double m = block_min(dtmin, sRed);
  if (tid == 0) a.cta_dt[blockIdx.x] = m;
}
