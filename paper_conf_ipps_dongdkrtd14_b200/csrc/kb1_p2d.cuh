// KB1 p2d — 2D corner force, persistent CTAs with the gather of the next zone batch in flight.
//
// Same mathematics and stages as kb1_corner_force_2d (kb1_corner_force.cuh; eq (4)-(6); DESIGN.md
// §1 rows a0-a5): stage A (a1 -> q1), the point evaluation (one thread per point), C^T, A^T.  What changes
// is the a0 row: kb1_corner_force_2d runs one zone batch per CTA and starts with a synchronous gather (a
// zone -> node id load, then the dependent x / v loads: two DRAM round trips before any arithmetic), so
// with ~2 waves of CTAs per SM that latency is exposed once per batch.  Here each CTA loops over batches
// b, b + grid, ... and copies batch b + grid (x, v through the node ids read one batch earlier; e;
// J0^{-1}; rho0|J0|; gamma) into the second of two prefetch buffers with cp.async while batch b computes.
// (C2, 2D Q4-Q3 64x64, is the config: ncu on kb1_corner_force_2d showed 20 % FP64 pipe and 28 % issue.)
#pragma once
#include "kb1_v2.cuh"

template <int K>
struct P2dDims {
  using D2 = Dims2<K>;
  static constexpr int N = D2::N, P = D2::P, T = D2::T, NK = D2::NK, NT = D2::NT, NQ = D2::NQ, NF = D2::NF;
  // prefetch block of one zone: X[NF][NK] E[NT] J0inv[4] R[NQ] gamma, padded to 16 bytes
  static constexpr int PF_X = 0, PF_E = NF * NK, PF_J = PF_E + NT, PF_R = PF_J + 4, PF_G = PF_R + NQ;
  static constexpr int PFZ = (PF_G + 1 + 1) / 2 * 2;
  // work block of one zone: T, S, Y (as kb1_corner_force_2d)
  static constexpr int WZ = D2::SZ_T + D2::SZ_S + D2::SZ_Y;
};

template <int K, int ZPC>
struct KB1CfgP2d {
  using Dm = P2dDims<K>;
  static constexpr int NTH = (ZPC * Dm::NQ + 31) / 32 * 32;
  static constexpr int TABP = (Dims2<K>::TAB + 1) / 2 * 2;
  static constexpr int SMEM_DOUBLES = TABP + 2 * ZPC * Dm::PFZ + ZPC * Dm::WZ + 32;
  static constexpr int SMEM_BYTES = SMEM_DOUBLES * 8;
  static constexpr int IDS = (ZPC * Dm::NK + NTH - 1) / NTH;   // node ids a thread prefetches per batch
};

template <int K, int ZPC, int MINB>
__global__ void __launch_bounds__(KB1CfgP2d<K, ZPC>::NTH, MINB) kb1_p2d(const KB1Args a) {
  using Dm = P2dDims<K>;
  using D2 = Dims2<K>;
  using Cfg = KB1CfgP2d<K, ZPC>;
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, NK = Dm::NK, NT = Dm::NT, NQ = Dm::NQ, NF = Dm::NF;
  constexpr int NTH = Cfg::NTH, IDS = Cfg::IDS;
  extern __shared__ double smem[];
  double *sB = smem, *sG = sB + N * P, *sPhi = sG + N * P, *sW = sPhi + N * T;
  double *sPF = smem + Cfg::TABP;                    // [2][ZPC][PFZ]
  double *sWork = sPF + 2 * ZPC * Dm::PFZ;           // [ZPC][WZ]: T | S | Y
  double *sRed = sWork + ZPC * Dm::WZ;

  const int tid0 = threadIdx.x;
  const int64_t Z = a.num_zones, nn = a.num_nodes;
  const int64_t nb = (Z + ZPC - 1) / ZPC, G = gridDim.x;

  int32_t ids[IDS];
  auto load_ids = [&](int64_t b, int tid) {
#pragma unroll
    for (int u = 0; u < IDS; ++u) {
      const int i = tid + u * NTH;
      const int64_t z = b * ZPC + i / NK;
      ids[u] = (i < ZPC * NK && b < nb && z < Z) ? __ldg(a.zone_nodes + b * ZPC * NK + i) : -1;
    }
  };
  auto issue = [&](int64_t b, double *pf, int tid) {   // batch b -> prefetch buffer pf (one commit group)
    if (b < nb) {
#pragma unroll
      for (int u = 0; u < IDS; ++u) {
        const int i = tid + u * NTH;
        if (i < ZPC * NK) {
          const int zl = i / NK, r = i - zl * NK;
          const bool v = ids[u] >= 0;
          const int64_t node = v ? ids[u] : 0;
          double *X = pf + zl * Dm::PFZ + Dm::PF_X + r;
#pragma unroll
          for (int c = 0; c < 2; ++c) {
            cp_async8(X + c * NK, a.x + c * nn + node, v);
            cp_async8(X + (2 + c) * NK, a.v + c * nn + node, v);
          }
        }
      }
      constexpr int PER = NT + 4 + NQ + 1;
      for (int i = tid; i < ZPC * PER; i += NTH) {
        const int zl = i / PER, r = i - zl * PER;
        const int64_t z = b * ZPC + zl;
        const bool v = z < Z;
        const int64_t zz = v ? z : 0;
        const double *src = r < NT ? a.e + zz * NT + r
                          : r < NT + 4 ? a.J0inv + zz * 4 + (r - NT)
                          : r < NT + 4 + NQ ? a.rho0detJ0 + zz * NQ + (r - NT - 4) : a.zone_gamma + zz;
        cp_async8(pf + zl * Dm::PFZ + Dm::PF_E + r, src, v);   // PF_E, PF_J, PF_R, PF_G are contiguous
      }
    }
    cp_async_commit();
  };

  for (int i = tid0; i < D2::TAB; i += NTH) smem[i] = __ldg(a.tab + i);
  int64_t b = blockIdx.x;
  load_ids(b, tid0);
  issue(b, sPF, tid0);
  load_ids(b + G, tid0);
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;

  for (int it = 0; b < nb; b += G, ++it) {
    int tid;   // re-read every batch (keeps the per-stage index arithmetic out of registers across the loop)
    asm volatile("mov.u32 %0, %%tid.x;" : "=r"(tid));
    const int cur = it & 1;
    const double *PF = sPF + cur * ZPC * Dm::PFZ;
    issue(b + G, sPF + (cur ^ 1) * ZPC * Dm::PFZ, tid);
    load_ids(b + 2 * G, tid);
    cp_async_wait<1>();
    __syncthreads();
    const int64_t zone0 = b * ZPC;

    // stage A: a1 -> q1 for every q1: TB[f][q1][a0] = sum_a1 B(q1,a1) X[f][a1][a0] (TG with G); TE
    for (int i = tid; i < ZPC * NF * N * P; i += NTH) {
      const int zl = i / (NF * N * P), rr = i - zl * (NF * N * P);
      const int f = rr / (N * P), r2 = rr - f * (N * P);
      const int qq1 = r2 / P, a0 = r2 - qq1 * P;
      const double *X = PF + zl * Dm::PFZ + Dm::PF_X + f * NK + a0;
      double tb = 0.0, tg = 0.0;
#pragma unroll
      for (int a1 = 0; a1 < P; ++a1) {
        tb = fma(sB[qq1 * P + a1], X[a1 * P], tb);
        tg = fma(sG[qq1 * P + a1], X[a1 * P], tg);
      }
      double *Tz = sWork + zl * Dm::WZ;
      Tz[f * N * P + r2] = tb;
      Tz[NF * N * P + f * N * P + r2] = tg;
    }
    for (int i = tid; i < ZPC * N * T; i += NTH) {
      const int zl = i / (N * T), r = i - zl * (N * T);
      const int qq1 = r / T, j0 = r - qq1 * T;
      const double *E = PF + zl * Dm::PFZ + Dm::PF_E;
      double te = 0.0;
#pragma unroll
      for (int j1 = 0; j1 < T; ++j1) te = fma(sPhi[qq1 * T + j1], E[j1 * T + j0], te);
      sWork[zl * Dm::WZ + 2 * NF * N * P + r] = te;
    }
    __syncthreads();

    // point evaluation: one thread per point
    const int my_zl = tid / NQ, my_q = tid - my_zl * NQ;
    const int q0 = my_q % N, q1 = my_q / N;
    const bool has_point = my_zl < ZPC;
    const int64_t my_z = zone0 + my_zl;
    const bool active = has_point && my_z < Z;
    if (has_point) {
      const double *Tz = sWork + my_zl * Dm::WZ;
      const double *pfz = PF + my_zl * Dm::PFZ;
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
      const double R = active ? pfz[Dm::PF_R + my_q] : 1.0;
      const double gamma = active ? pfz[Dm::PF_G] : 1.4;
      const double J0i[4] = {pfz[Dm::PF_J + 0], pfz[Dm::PF_J + 1], pfz[Dm::PF_J + 2], pfz[Dm::PF_J + 3]};
      PointOut<2> o;
      point_eval2(Jm, Gv, eq, R, sW[q0] * sW[q1], gamma, J0i, a.ph, o);
      double *S = sWork + my_zl * Dm::WZ + D2::SZ_T;
#pragma unroll
      for (int c = 0; c < 2; ++c)
#pragma unroll
        for (int d = 0; d < 2; ++d) S[(c * 2 + d) * NQ + my_q] = o.S[c][d];
      S[4 * NQ + my_q] = o.P;
      if (a.Sq != nullptr && active) {
#pragma unroll
        for (int c = 0; c < 4; ++c) a.Sq[(my_z * NQ + my_q) * 4 + c] = o.S[c / 2][c % 2];
      }
      if (active) {
        dtmin = fmin(dtmin, o.dt);
        bad |= o.bad;
      }
    }
    __syncthreads();

    // C^T: Y[c][0][q1][a0] = sum_q0 G(q0,a0) S_c0 ; Y[c][1][q1][a0] = sum_q0 B(q0,a0) S_c1 ; YE
    for (int i = tid; i < ZPC * 2 * N * P; i += NTH) {
      const int zl = i / (2 * N * P), rr = i - zl * (2 * N * P);
      const int c = rr / (N * P), r2 = rr - c * (N * P);
      const int qq1 = r2 / P, a0 = r2 - qq1 * P;
      const double *S = sWork + zl * Dm::WZ + D2::SZ_T + qq1 * N;
      double y0 = 0.0, y1 = 0.0;
#pragma unroll
      for (int qq0 = 0; qq0 < N; ++qq0) {
        y0 = fma(sG[qq0 * P + a0], S[(c * 2 + 0) * NQ + qq0], y0);
        y1 = fma(sB[qq0 * P + a0], S[(c * 2 + 1) * NQ + qq0], y1);
      }
      double *Y = sWork + zl * Dm::WZ + D2::SZ_T + D2::SZ_S + c * 2 * N * P;
      Y[r2] = y0;
      Y[N * P + r2] = y1;
    }
    for (int i = tid; i < ZPC * N * T; i += NTH) {
      const int zl = i / (N * T), r = i - zl * (N * T);
      const int qq1 = r / T, j0 = r - qq1 * T;
      const double *Pz = sWork + zl * Dm::WZ + D2::SZ_T + 4 * NQ + qq1 * N;
      double ye = 0.0;
#pragma unroll
      for (int qq0 = 0; qq0 < N; ++qq0) ye = fma(sPhi[qq0 * T + j0], Pz[qq0], ye);
      sWork[zl * Dm::WZ + D2::SZ_T + D2::SZ_S + 4 * N * P + r] = ye;
    }
    __syncthreads();

    // A^T: (F_z 1)[c][a1][a0] = sum_q1 B(q1,a1) Y[c][0][q1][a0] + G(q1,a1) Y[c][1][q1][a0]; F^T v
    for (int i = tid; i < ZPC * 2 * NK; i += NTH) {
      const int zl = i / (2 * NK), rr = i - zl * (2 * NK);
      const int c = rr / NK, r = rr - c * NK;
      const int a1 = r / P, a0 = r - a1 * P;
      const double *Y = sWork + zl * Dm::WZ + D2::SZ_T + D2::SZ_S + c * 2 * N * P + a0;
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
      const double *YE = sWork + zl * Dm::WZ + D2::SZ_T + D2::SZ_S + 4 * N * P + j0;
      double s = 0.0;
#pragma unroll
      for (int qq1 = 0; qq1 < N; ++qq1) s = fma(sPhi[qq1 * T + j1], YE[qq1 * T], s);
      if (zone0 + zl < Z) a.FTv[zone0 * NT + i] = s;
    }
    // (the next batch's stage A writes T after this batch's C^T barrier; its prefetch buffer was last read
    // in this batch's point stage, before that barrier)
  }
  cp_async_wait<0>();
  if (bad) dtmin = 0.0;
  const double m = block_min(dtmin, sRed);
  if (tid0 == 0) a.cta_dt[blockIdx.x] = m;
}
