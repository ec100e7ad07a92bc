// KB1 v6 — warp-specialized 3D corner force (k = 4) with the contraction warps on DFMA, not DMMA.
//
// Same mathematics and buffers as kb1_v5.cuh (eq (4)-(6); DESIGN.md §1 rows a0-a5): point
// warps PW run stage C of the velocity fields, e(q) and the point physics of zone i; contraction warps
// KW run the back stages of zone i-1 and the gather + forward stages (A, B, and C for the position
// fields, i.e. J) of zone i+1; J in / S out share the in-place JS buffer.
//
// Why DFMA here (tools/pipe_share.cu, profiles/r01_pipe_share.txt): DFMA and DMMA issue into ONE FP64
// pipe on sm_100a, and a stream of DMMAs (16 pipe cycles each per SMSP) starves concurrent DFMA warps
// completely.  PW is latency-bound (alone: 8.1 K cycles/zone for 4.6 K pipe cycles of work), so every
// DMMA the contraction warps issue lands on PW's critical path: v5 measured PW alone 8.1 K, KW alone
// 8.5 K, together 13.2 K cycles per zone.  As DFMA the contractions (a) need no padding (p = 5 is not a
// multiple of the MMA k = 4: 1.6x fewer pipe cycles), (b) occupy the pipe in 2-cycle quanta that
// interleave with PW's dependent chains, and (c) have high ILP (8-24 independent accumulators per
// thread), so they fill the pipe cycles PW leaves idle instead of blocking it.  The 1-D tables are
// constant-bank operands with compile-time indices (kb1_v2.cuh's CT<K>), so a contraction stage is
// LDS -> DFMA c[][] -> STS with no table loads.
//
// JS layout: J/S of point (col = q2*N + q1, q0) at col*8 + 2*((q0/2) ^ g(col)) + (q0 & 1) (js_idx): the
// pair swizzle makes the contraction warps' 16-byte row accesses (8 consecutive cols, one q0 pair) and
// the point warps' 8-byte accesses (4 q0 x 8 q1 per warp) both conflict-free.
#pragma once
#include "kb1_v5.cuh"

// Pair slot of q0 in row col: (q0/2) ^ g(col), g = the 2-bit reversal of (col/2) & 3.  g is a bijection, so the
// contraction warps' 16-byte row accesses (8 consecutive rows, one pair) stay conflict-free, and
// g(1) ^ g(0) = g(3) ^ g(2) = 2, so the 8-byte accesses of a half-warp (rows c..c+3 of one slab x 4 q0: the
// point warps and the DMMA fragments of kb1_v10.cuh) fill 16 distinct banks.  (The first form, (q0/2) ^
// (col/2), left those 2-way conflicted: ncu on v10, profiles/r01_kw_stage_clocks.txt.)
__device__ __forceinline__ int js_idx(int col, int q0) {
  const int g = (col & 2) | ((col >> 2) & 1);   // 2-bit reversal of (col / 2) & 3
  return col * 8 + ((((q0 >> 1) ^ g) & 3) << 1) + (q0 & 1);
}
__device__ __forceinline__ void lds_f64x2(const double *src, double &a, double &b) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(src);
  asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];\n" : "=d"(a), "=d"(b) : "r"(s) : "memory");
}

// The 1-D tables come from the constant bank (uniform LDCU feeding DFMA's uniform-register operand) at
// an offset o that is always 0 but not provably so (zone >> 40, >> 41, ...): the loads stay inside the
// zone loop and are not shared between the work-item blocks of a stage.  Plain C.B(q, a) reads are
// loop-invariant, get hoisted into ordinary registers and spill the 88-register contraction warps (the
// tables are 112 doubles).  For the same reason every stage is straight-line code (at most 3 work
// items per thread, each block with its own offset) instead of a loop over work items.
template <int K>
struct CTZ {
  static constexpr int N = 2 * K, P = K + 1, T = K, OFF = ctab_off(K);
  int o;
  __device__ __forceinline__ double B(int q, int a) const { return c_tabs[OFF + o + q * P + a]; }
  __device__ __forceinline__ double G(int q, int a) const { return c_tabs[OFF + o + N * P + q * P + a]; }
  __device__ __forceinline__ double Phi(int q, int j) const { return c_tabs[OFF + o + 2 * N * P + q * T + j]; }
};

template <int K, int DIAG = 0>
__global__ void __launch_bounds__(KB1V5Cfg<K>::NTH, 1) kb1_v6_3d(const KB1Args a) {
  using Dm = V5Dims<K>;
  using Cfg = KB1V5Cfg<K>;
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, P2 = Dm::P2, P3 = Dm::P3, T2 = Dm::T2, T3 = Dm::T3;
  constexpr int N2 = Dm::N2, N3 = Dm::N3, NH = Dm::NH, TPZ = Dm::TPZ;
  constexpr int NPW = Cfg::NPW, NKW = Cfg::NKW;
  static_assert(NKW >= P3, "the gather gives one node per contraction-warp thread");
  static_assert(N == 8, "kb1_v6: the JS swizzle is written for lines of 8 points");
  extern __shared__ double smem[];
  double *sTab = smem;
  const double *tB = sTab, *tG = sTab + N * P, *tPhi = sTab + 2 * N * P, *sW = sTab + 2 * N * P + N * T;
  double *sJS = smem + Dm::OFF_JS, *sUV = smem + Dm::OFF_UV, *sXE = smem + Dm::OFF_XE, *sWk = smem + Dm::OFF_W;
  double *sJ = smem + Dm::OFF_J, *sRed = smem + Dm::OFF_RED;

  const int tid = threadIdx.x;
  const bool is_kw = tid >= NPW;
  const int ktid = tid - NPW;
  const int64_t Z = a.num_zones, nn = a.num_nodes;
  const int64_t G = gridDim.x;
  const int64_t nz = Z > blockIdx.x ? (Z - 1 - blockIdx.x) / G + 1 : 0;
  auto zone_of = [&](int64_t i) { return (int64_t)blockIdx.x + i * G; };
  // stage clocks of the contraction warps (a.prof != nullptr only): sKP[s] accumulates the cycles of
  // stage s, sKP[15] holds the last stamp; written by KW thread 0 alone (PW's dt reduction uses sRed[0, 16))
  long long *sKP = reinterpret_cast<long long *>(smem + Dm::OFF_RED + 16);
  auto kstamp = [&](int slot) {
    if (a.prof != nullptr && tid == NPW) {
      const long long t = clock64();
      sKP[slot] += t - sKP[15];
      sKP[15] = t;
    }
  };

  for (int i = tid; i < 2 * N * P + N * T + N; i += Cfg::NTH) sTab[i] = __ldg(a.tab + i);
  if (tid == 0) sRed[8] = 0.0;   // dt filter: best exact inverse dt of this CTA (point_eval3<true>)

  // ---------------- KW ----------------
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
  auto kw_forward = [&](double *ub, double *jb, double *js, int zc) {
    const int kt = opaque_tid() - NPW;
    if (kt < 10) js[kt] = sXE[Dm::XE_J + kt];
    double *Tr = sWk, *UX = sWk + Dm::O_UX;
    // stage A: a2 -> q2 (T_B, T_G of the 6 fields; TE of e)
    {
    const int r0_ = kt;
#pragma unroll
    for (int blk = 0; blk < (6 * P2 + T2 + NKW - 1) / NKW; ++blk) {
      const int r = r0_ + blk * NKW;
      const CTZ<K> C{zc * (blk + 1)};
      if (r < 6 * P2 + T2) {
      if (r < 6 * P2) {
        const int f = r / P2, aa = r - f * P2;
        double xv[P];
#pragma unroll
        for (int a2 = 0; a2 < P; ++a2) xv[a2] = sXE[Dm::XE_X + f * P3 + a2 * P2 + aa];
        double *TB = Tr + Dm::O_T + (f * 2 + 0) * N * P2 + aa, *TG = TB + N * P2;
#pragma unroll
        for (int q2 = 0; q2 < N; ++q2) {
          double tb = 0.0, tg = 0.0;
#pragma unroll
          for (int a2 = 0; a2 < P; ++a2) {
            tb = fma(C.B(q2, a2), xv[a2], tb);
            tg = fma(C.G(q2, a2), xv[a2], tg);
          }
          TB[q2 * P2] = tb;
          TG[q2 * P2] = tg;
        }
      } else {
        const int jj = r - 6 * P2;
        double ev[T];
#pragma unroll
        for (int j2 = 0; j2 < T; ++j2) ev[j2] = sXE[Dm::XE_E + j2 * T2 + jj];
#pragma unroll
        for (int q2 = 0; q2 < N; ++q2) {
          double te = 0.0;
#pragma unroll
          for (int j2 = 0; j2 < T; ++j2) te = fma(C.Phi(q2, j2), ev[j2], te);
          Tr[Dm::O_TE + q2 * T2 + jj] = te;
        }
      }
    }}}
    kw_bar<NKW>();
    kstamp(8);
    // stage B: a1 -> q1; position fields -> UX (scratch), velocity fields + e -> ub
    {
    const int r0_ = opaque_tid() - NPW;
#pragma unroll
    for (int blk = 0; blk < (6 * N * P + N * T + NKW - 1) / NKW; ++blk) {
      const int r = r0_ + blk * NKW;
      const CTZ<K> C{zc * (blk + 1)};
      if (r < 6 * N * P + N * T) {
      if (r < 6 * N * P) {
        const int f = r / (N * P), r2 = r - f * (N * P), q2 = r2 / P, a0 = r2 - q2 * P;
        double tb[P], tg[P];
#pragma unroll
        for (int a1 = 0; a1 < P; ++a1) {
          tb[a1] = Tr[Dm::O_T + ((f * 2 + 0) * N + q2) * P2 + a1 * P + a0];
          tg[a1] = Tr[Dm::O_T + ((f * 2 + 1) * N + q2) * P2 + a1 * P + a0];
        }
        double *U0 = (f < 3 ? UX + f * 3 * N2 * P : ub + (f - 3) * 3 * N2 * P) + q2 * N * P + a0;
#pragma unroll
        for (int q1 = 0; q1 < N; ++q1) {
          double u0 = 0.0, u1 = 0.0, u2 = 0.0;
#pragma unroll
          for (int a1 = 0; a1 < P; ++a1) {
            u0 = fma(C.B(q1, a1), tb[a1], u0);
            u1 = fma(C.G(q1, a1), tb[a1], u1);
            u2 = fma(C.B(q1, a1), tg[a1], u2);
          }
          U0[q1 * P] = u0;
          U0[N2 * P + q1 * P] = u1;
          U0[2 * N2 * P + q1 * P] = u2;
        }
      } else {
        const int r2 = r - 6 * N * P, q2 = r2 / T, j0 = r2 - q2 * T;
        double te[T];
#pragma unroll
        for (int j1 = 0; j1 < T; ++j1) te[j1] = Tr[Dm::O_TE + q2 * T2 + j1 * T + j0];
#pragma unroll
        for (int q1 = 0; q1 < N; ++q1) {
          double ue = 0.0;
#pragma unroll
          for (int j1 = 0; j1 < T; ++j1) ue = fma(C.Phi(q1, j1), te[j1], ue);
          ub[Dm::O_UE + (q2 * N + q1) * T + j0] = ue;
        }
      }
    }}}
    kw_bar<NKW>();
    kstamp(9);
    // stage C (position fields): J[c][m](col, q0) = sum_a0 M_m[q0][a0] UX[c][m][col][a0] -> JS (swizzled)
    {
    const int r0_ = opaque_tid() - NPW;
#pragma unroll
    for (int blk = 0; blk < (9 * N2 + NKW - 1) / NKW; ++blk) {
      const int r = r0_ + blk * NKW;
      const CTZ<K> C{zc * (blk + 1)};
      if (r < 9 * N2) {
      const int cm = r / N2, col = r - cm * N2;   // cm is warp-uniform (N2 = 64)
      double uv[P];
#pragma unroll
      for (int a0 = 0; a0 < P; ++a0) uv[a0] = UX[cm * N2 * P + col * P + a0];
      double o[N];
      if (cm % 3 == 0) {
#pragma unroll
        for (int q0 = 0; q0 < N; ++q0) {
          double s = 0.0;
#pragma unroll
          for (int a0 = 0; a0 < P; ++a0) s = fma(C.G(q0, a0), uv[a0], s);
          o[q0] = s;
        }
      } else {
#pragma unroll
        for (int q0 = 0; q0 < N; ++q0) {
          double s = 0.0;
#pragma unroll
          for (int a0 = 0; a0 < P; ++a0) s = fma(C.B(q0, a0), uv[a0], s);
          o[q0] = s;
        }
      }
      double *dst = jb + cm * N3;
#pragma unroll
      for (int pq = 0; pq < N / 2; ++pq) sts_f64x2(dst + js_idx(col, 2 * pq), o[2 * pq], o[2 * pq + 1]);
    }}}
    kstamp(10);
  };
  auto kw_back = [&](const double *sb, int64_t z, int zc) {
    double *Wr = sWk;
    // C^T: q0 -> a0 for the 9 S components (3 items per col) and Pq
    {
    const int r0_ = opaque_tid() - NPW;
#pragma unroll
    for (int blk = 0; blk < (4 * N2 + NKW - 1) / NKW; ++blk) {
      const int r = r0_ + blk * NKW;
      const CTZ<K> C{zc * (blk + 1)};
      if (r < 4 * N2) {
      const int c = r / N2, col = r - c * N2;   // warp-uniform c
      if (c < 3) {
#pragma unroll
        for (int d = 0; d < 3; ++d) {   // one S component at a time (register budget of the KW warps)
          double sv[N];
          const double *bd = sb + (c * 3 + d) * N3;
#pragma unroll
          for (int pq = 0; pq < N / 2; ++pq) lds_f64x2(bd + js_idx(col, 2 * pq), sv[2 * pq], sv[2 * pq + 1]);
#pragma unroll
          for (int a0 = 0; a0 < P; ++a0) {
            double y = 0.0;
#pragma unroll
            for (int q0 = 0; q0 < N; ++q0) y = fma(d == 0 ? C.G(q0, a0) : C.B(q0, a0), sv[q0], y);
            Wr[Dm::O_Y + ((c * 3 + d) * P + a0) * N2 + col] = y;
          }
        }
      } else {
        double pv[N];
#pragma unroll
        for (int pq = 0; pq < N / 2; ++pq) lds_f64x2(sb + Dm::O_PQ + js_idx(col, 2 * pq), pv[2 * pq], pv[2 * pq + 1]);
#pragma unroll
        for (int j0 = 0; j0 < T; ++j0) {
          double y = 0.0;
#pragma unroll
          for (int q0 = 0; q0 < N; ++q0) y = fma(C.Phi(q0, j0), pv[q0], y);
          Wr[Dm::O_YE + j0 * N2 + col] = y;
        }
      }
    }}}
    kw_bar<NKW>();
    kstamp(4);
    // B^T: q1 -> a1
    {
    const int r0_ = opaque_tid() - NPW;
#pragma unroll
    for (int blk = 0; blk < (3 * P * N + T * N + NKW - 1) / NKW; ++blk) {
      const int r = r0_ + blk * NKW;
      const CTZ<K> C{zc * (blk + 1)};
      if (r < 3 * P * N + T * N) {
      if (r < 3 * P * N) {
        const int c = r / (P * N), r2 = r - c * (P * N), a0 = r2 / N, q2 = r2 - a0 * N;
        const double *Yb = Wr + Dm::O_Y + ((c * 3) * P + a0) * N2 + q2 * N;
        {   // zb = B^T y0 + G^T y1
          double y0[N], y1[N];
#pragma unroll
          for (int q1 = 0; q1 < N; ++q1) { y0[q1] = Yb[q1]; y1[q1] = Yb[P * N2 + q1]; }
#pragma unroll
          for (int a1 = 0; a1 < P; ++a1) {
            double zb = 0.0;
#pragma unroll
            for (int q1 = 0; q1 < N; ++q1) {
              zb = fma(C.B(q1, a1), y0[q1], zb);
              zb = fma(C.G(q1, a1), y1[q1], zb);
            }
            Wr[Dm::O_Z + ((c * 2 + 0) * N + q2) * P2 + a1 * P + a0] = zb;
          }
        }
        {   // zg = B^T y2
          double y2[N];
#pragma unroll
          for (int q1 = 0; q1 < N; ++q1) y2[q1] = Yb[2 * P * N2 + q1];
#pragma unroll
          for (int a1 = 0; a1 < P; ++a1) {
            double zg = 0.0;
#pragma unroll
            for (int q1 = 0; q1 < N; ++q1) zg = fma(C.B(q1, a1), y2[q1], zg);
            Wr[Dm::O_Z + ((c * 2 + 1) * N + q2) * P2 + a1 * P + a0] = zg;
          }
        }
      } else {
        const int r2 = r - 3 * P * N, j0 = r2 / N, q2 = r2 - j0 * N;
        double ye[N];
#pragma unroll
        for (int q1 = 0; q1 < N; ++q1) ye[q1] = Wr[Dm::O_YE + j0 * N2 + q2 * N + q1];
#pragma unroll
        for (int j1 = 0; j1 < T; ++j1) {
          double ze = 0.0;
#pragma unroll
          for (int q1 = 0; q1 < N; ++q1) ze = fma(C.Phi(q1, j1), ye[q1], ze);
          Wr[Dm::O_ZE + q2 * T2 + j1 * T + j0] = ze;
        }
      }
    }}}
    kw_bar<NKW>();
    kstamp(5);
    // A^T: q2 -> a2, straight to global
    {
    const int r0_ = opaque_tid() - NPW;
#pragma unroll
    for (int blk = 0; blk < (3 * P2 + T2 + NKW - 1) / NKW; ++blk) {
      const int r = r0_ + blk * NKW;
      const CTZ<K> C{zc * (blk + 1)};
      if (r < 3 * P2 + T2) {
      if (r < 3 * P2) {
        const int c = r / P2, aa = r - c * P2;
        double zb[N], zg[N];
#pragma unroll
        for (int q2 = 0; q2 < N; ++q2) {
          zb[q2] = Wr[Dm::O_Z + ((c * 2 + 0) * N + q2) * P2 + aa];
          zg[q2] = Wr[Dm::O_Z + ((c * 2 + 1) * N + q2) * P2 + aa];
        }
#pragma unroll
        for (int a2 = 0; a2 < P; ++a2) {
          double s = 0.0;
#pragma unroll
          for (int q2 = 0; q2 < N; ++q2) {
            s = fma(C.B(q2, a2), zb[q2], s);
            s = fma(C.G(q2, a2), zg[q2], s);
          }
          a.Fz1[(z * 3 + c) * P3 + a2 * P2 + aa] = s;
        }
      } else {
        const int jj = r - 3 * P2;
        double ze[N];
#pragma unroll
        for (int q2 = 0; q2 < N; ++q2) ze[q2] = Wr[Dm::O_ZE + q2 * T2 + jj];
#pragma unroll
        for (int j2 = 0; j2 < T; ++j2) {
          double s = 0.0;
#pragma unroll
          for (int q2 = 0; q2 < N; ++q2) s = fma(C.Phi(q2, j2), ze[q2], s);
          a.FTv[z * T3 + j2 * T2 + jj] = s;
        }
      }
    }}}
    kw_bar<NKW>();   // Y/Z scratch free again
    kstamp(6);
  };

  // ---------------- PW ----------------
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;
  const int pr = tid, q0a = pr % NH, q1 = (pr / NH) % N, q2 = pr / (NH * N);
  auto pw_point = [&](const double *ub, const double *js, double *jb, int64_t z) {
    const double gamma = js[9];
    const int col = q2 * N + q1;
    const int qa = col * N + q0a, qb = qa + NH;                     // natural point index (R, Sq)
    const int sa = js_idx(col, q0a), sbi = js_idx(col, q0a + NH);  // JS slots
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
      const double ue = ub[Dm::O_UE + col * T + j0];
      ea = fma(tPhi[q0a * T + j0], ue, ea);
      eb = fma(tPhi[(q0a + NH) * T + j0], ue, eb);
    }
    double Ja[3][3], Gva[3][3], Jb[3][3], Gvb[3][3];
#pragma unroll
    for (int c = 0; c < 3; ++c)
#pragma unroll
      for (int d = 0; d < 3; ++d) {
        Ja[c][d] = jb[(c * 3 + d) * N3 + sa]; Gva[c][d] = ga[c * 3 + d];
        Jb[c][d] = jb[(c * 3 + d) * N3 + sbi]; Gvb[c][d] = gb[c * 3 + d];
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
    for (int cd = 0; cd < 9; ++cd) {     // in place over J: only this thread touches slots sa, sbi
      jb[cd * N3 + sa] = oa.S[cd / 3][cd % 3];
      jb[cd * N3 + sbi] = ob.S[cd / 3][cd % 3];
    }
    jb[Dm::O_PQ + sa] = oa.P;
    jb[Dm::O_PQ + sbi] = ob.P;
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
    if (nz > 0 && DIAG != 1) kw_forward(sUV, sJS, sJ, a.zero);
    __syncthreads();
    long long t_work = 0;
    int itc = 2;
    for (int64_t i = 0; i <= nz; ++i, ++itc) {
      const long long t0 = clock64();
      kw_issue(i + 1);
      kw_load_id(i + 2);
      cp_async_commit();
      kstamp(3);
      const int zc = a.zero * itc;   // 0, but loop-variant and uniform
      if (i >= 1 && DIAG != 1) kw_back(sJS + ((i - 1) & 1) * Dm::JSBUF, zone_of(i - 1), zc);
      cp_async_wait<0>();
      kw_bar<NKW>();
      kstamp(7);
      if (i + 1 < nz && DIAG != 1)
        kw_forward(sUV + ((i + 1) & 1) * Dm::UVBUF, sJS + ((i + 1) & 1) * Dm::JSBUF, sJ + ((i + 1) & 1) * 10, zc + a.zero);
      t_work += clock64() - t0;
      __syncthreads();
      kstamp(11);
    }
    if (a.prof != nullptr && tid == NPW) {
      a.prof[blockIdx.x * 16 + 1] = t_work;
      for (int sl = 3; sl < 12; ++sl) a.prof[blockIdx.x * 16 + sl] = sKP[sl];
    }
    return;
  }
  asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;\n" ::"n"(Cfg::REG_PW));
  __syncthreads();
  long long t_work = 0, t_all = clock64();
  for (int64_t i = 0; i <= nz; ++i) {
    const long long t0 = clock64();
    if (i < nz && tid < TPZ && DIAG != 2)
      pw_point(sUV + (i & 1) * Dm::UVBUF, sJ + (i & 1) * 10, sJS + (i & 1) * Dm::JSBUF, zone_of(i));
    t_work += clock64() - t0;
    __syncthreads();
  }
  if (a.prof != nullptr && tid == 0) {
    a.prof[blockIdx.x * 16 + 0] = t_work;
    a.prof[blockIdx.x * 16 + 2] = clock64() - t_all;
  }
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
