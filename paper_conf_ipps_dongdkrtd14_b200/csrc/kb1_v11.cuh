// KB1 v11 — persistent 3D corner force for high orders (k = 7, 8; C5 is k = 8): kb1_v8.cuh's per-slab
// stages, with the two costs ncu attributed to v8 (gpurun_out c5_v8 capture) removed:
//   * the gather of every zone stalled all warps at the start of the CTA (13 % of the warp-stall samples:
//     node ids -> coordinates, dependent DRAM loads).  v11 is persistent (2 CTAs per SM walk zones
//     z = blockIdx.x + i * gridDim.x) and gathers zone i+1 by cp.async into sX / sE right after stage A of
//     zone i's LAST slab (the only reader of sX / sE), so the copies fly under the remaining five stages
//     of that slab; the next zone's node ids and e are prefetched into L2 at its first slab;
//   * stage B^T ran on 3 of 8 warps (up to 288 DFMA per thread while 5 warps waited at the barrier):
//     v11 splits every B^T item's a1 outputs over warps so all 8 warps work (at most 32 loads + 96 DFMA).
// Mathematics, slab order, summation orders and outputs are those of v8 (eq (4)-(6); DESIGN.md
// §1 rows a0-a5); J0^{-1} and gamma are double-buffered (the point stage of the last slab still reads
// zone i's while zone i+1's arrive).
#pragma once
#include "kb1_v8.cuh"

template <int K>
struct V11Dims : V8Dims<K> {
  using B = V8Dims<K>;
  // O_J0 region grows from 10 to 20 doubles (two buffers of J0^{-1}[9] + gamma)
  static constexpr int FIX = (B::O_J0 + 20 + 1) / 2 * 2;
  static constexpr int OFF_FIX = B::TAB, OFF_A = OFF_FIX + FIX, OFF_B = OFF_A + (B::RA + 1) / 2 * 2;
  static constexpr int OFF_RED = OFF_B + (B::RB + 1) / 2 * 2;
  static constexpr int TOTAL = OFF_RED + 32;
};

template <int K>
struct KB1V11Cfg {
  using Dm = V11Dims<K>;
  static constexpr int NTH = (Dm::NS + 31) / 32 * 32;
  static constexpr int SMEM_BYTES = Dm::TOTAL * 8;
};

// MB = 1: stage B on DMMA (mma.sync m8n8k4 f64): U_X[q1][col] = sum_a1 X[q1][a1] In[a1][col] for the tables
// X = B (columns: the TB and TG lines of the 6 fields, 108) and X = G (the TB lines, 54), K = P padded to a
// multiple of 4, plus the e lines with Phi (K = T): 22 n-tiles of 8 columns over the 8 warps.  One DMMA does
// 256 FMAs (the DFMA form issues an LDCU of the table coefficient next to every DFMA).
template <int K, int MINB, int MB = 0>
__global__ void __launch_bounds__(KB1V11Cfg<K>::NTH, MINB) kb1_v11_3d(const KB1Args a) {
  using Dm = V11Dims<K>;
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, P2 = Dm::P2, NK = Dm::NK, NT = Dm::NT, NS = Dm::NS;
  constexpr int T2 = Dm::T2, PP = Dm::PP, SR = Dm::SR;
  constexpr int NTH = KB1V11Cfg<K>::NTH;
  constexpr bool FILTER = NS % 32 == 0;   // every warp full of points: the dt filter's vote is legal
  static_assert(NTH >= 192, "stage C^T: six warps of row items (k >= 7)");
  static_assert(NTH >= 6 * 3 * P + T, "stage B: one item per thread");
  static_assert(NTH >= 3 * P2, "stage A^T: one item per thread");
  static_assert(P % 3 == 0 || P == 8, "stage B^T: a1 split in three parts of P/3 (k = 8) or two of 4 (k = 7)");
  static_assert(3 * P <= 32, "stage B^T: one (c, a0) item per lane");
  constexpr int NPART = P % 3 == 0 ? 3 : 2, PL = P / NPART;   // B^T: a1 parts per item
  // MB bit 4 (SDT): the CTA's min dt is kept in shared memory (one warp-min + atomicMin per warp and slab)
  // instead of a register pair + flag live across the whole zone loop.  At the 128-register cap those were
  // spilled and reloaded in stages A and C, whose loads then missed the small L1 (2 CTAs x ~100 KB of shared
  // memory per SM): ncu put 7 % of v11.mbt's stall samples on those reloads (long scoreboard).  48 -> 24 B
  // of spills (what is left sits inside the eigen-solve), 13.73 -> 12.88 ms on C5.
  constexpr bool SDT = MB & 16;
  extern __shared__ double smem[];
  double *sB = smem, *sG = sB + N * P, *sPhi = sG + N * P, *sW = sPhi + N * Dm::TS;
  double *sF = smem + Dm::OFF_FIX;
  double *sX = sF + Dm::O_X, *sE = sF + Dm::O_E, *sAF = sF + Dm::O_AF, *sAE = sF + Dm::O_AE, *sJ0b = sF + Dm::O_J0;
  double *sA = smem + Dm::OFF_A, *sBr = smem + Dm::OFF_B, *sRed = smem + Dm::OFF_RED;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t Z = a.num_zones, nn = a.num_nodes, G = gridDim.x;
  // MB bit 6 (I32): the zone loop counter in 32 bits (fewer registers live across the point stage; zone
  // offsets are still formed in 64 bits)
  using ZI = typename std::conditional<(MB & 64) != 0, int, int64_t>::type;
  const ZI nz = (ZI)(Z > blockIdx.x ? (Z - 1 - blockIdx.x) / G + 1 : 0);
  auto zone_of = [&](int64_t i) { return (int64_t)blockIdx.x + i * G; };

  // gather of zone i (cp.async; the caller commits / waits): X, V [6][NK], e [NT], J0^{-1} + gamma
  auto gather = [&](int64_t i) {
    const int64_t z = zone_of(i);
    for (int r = tid; r < NK; r += NTH) {
      const int64_t node = __ldg(a.zone_nodes + z * NK + r);
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        cp_async8(sX + c * NK + r, a.x + c * nn + node, true);
        cp_async8(sX + (3 + c) * NK + r, a.v + c * nn + node, true);
      }
    }
    for (int r = tid; r < NT; r += NTH) cp_async8(sE + r, a.e + z * NT + r, true);
    if (tid < 10) cp_async8(sJ0b + (i & 1) * 10 + tid, tid < 9 ? a.J0inv + z * 9 + tid : a.zone_gamma + z, true);
  };

  // ---- tables, zone 0's gather, accumulators ------------------------------------------------------
  for (int i = tid; i < 2 * N * P + N * T + N; i += NTH) {   // B, G; Phi into rows of TS; W
    const double t = __ldg(a.tab + i);
    if (i < 2 * N * P) smem[i] = t;
    else if (i < 2 * N * P + N * T) sPhi[((i - 2 * N * P) / T) * Dm::TS + (i - 2 * N * P) % T] = t;
    else sW[i - 2 * N * P - N * T] = t;
  }
  for (int r = tid; r < 3 * NK; r += NTH) sAF[r] = 0.0;
  for (int r = tid; r < NT; r += NTH) sAE[r] = 0.0;
  if (tid == 0) sRed[8] = 0.0;   // dt filter: the CTA's best exact inverse dt
  if (SDT && tid == 0) sRed[10] = __longlong_as_double(0x7ff0000000000000LL);   // SDT: the CTA's min dt
  if (nz > 0) gather(0);
  cp_async_commit();
  cp_async_wait<0>();
  __syncthreads();

  const int q0 = tid % N, q1 = tid / N;
  const bool has_point = tid < NS;
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;

#pragma unroll 1
  for (ZI zi = 0; zi < nz; ++zi) {
    const int64_t z = zone_of(zi);
    const double *sJ0 = sJ0b + (zi & 1) * 10;
    const bool more = zi + 1 < nz;
#pragma unroll 1
    for (int q2 = 0; q2 < N; ++q2) {
      const int o = a.zero * (q2 + 1);   // 0, but loop-variant and uniform: the table loads stay here
      if (has_point)
        asm volatile("prefetch.global.L1 [%0];" ::"l"(a.rho0detJ0 + z * (int64_t)(N * NS) + (q2 * N + q1) * N + q0));
      if (q2 == 0 && more) {   // the next zone's node ids and e into L2, 15 slabs ahead of their use
        const int64_t z1 = zone_of(zi + 1);
        if (tid * 32 < NK) asm volatile("prefetch.global.L2 [%0];" ::"l"(a.zone_nodes + z1 * NK + tid * 32));
        if (tid * 16 < NT) asm volatile("prefetch.global.L2 [%0];" ::"l"(a.e + z1 * NT + tid * 16));
      }
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
            if (MB) {   // [a1][108] lines: TB of the 6 fields (f, a0) in columns 0..53, TG in 54..107
              const int a1 = rr / P, a0 = rr - a1 * P;
              sA[a1 * 108 + f * P + a0] = tb;
              sA[a1 * 108 + 54 + f * P + a0] = tg;
            } else {
              sA[f * P2 + rr] = tb;
              sA[6 * P2 + f * P2 + rr] = tg;
            }
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
      // last slab: sX / sE are dead -> gather the next zone under the remaining stages of this slab
      if (q2 == N - 1 && more) {
        gather(zi + 1);
        cp_async_commit();
      }
      // ---- stage B: a1 -> q1; item (f, m, a0) produces U[f][m][q1 = 0..N-1][a0] --------------------
      if (MB) {
        static_assert(!MB || (N == 16 && NTH == 256), "DMMA stage B is written for k = 8 (two m-tiles of q1)");
        constexpr int KSP = (P + 3) / 4, KST = (T + 3) / 4;       // k-steps of the B/G and Phi contractions
        constexpr int NB = (108 + 7) / 8, NG = (54 + 7) / 8;      // n-tiles of the B-table and G-table columns
        constexpr int NTILE = NB + NG + 1;                          // + one tile of the 8 e lines
        const int lr = lane >> 2, lc = lane & 3;
        static_assert(!MB || 6 * P == 54, "the [a1][108] T layout");
        // MB bit 8 (TBW): warps 0-4 take the 14 B-table tiles, warps 5-7 the 7 G-table tiles and the Phi tile, so a
        // warp's A fragments (its table's rows 8 mt + lr, k = 4 ks + lc) are loaded from shared memory once per slab
        // instead of once per tile (those loads were 11 % of the kernel's shared wavefronts, 45 % of them bank-conflict
        // excess: row stride P = 9)
        constexpr bool TBW = MB & 256;
        const int ptab = warp < 5 ? 0 : 1;
        double afr[2][KSP];
#pragma unroll
        for (int mt = 0; mt < 2; ++mt)
#pragma unroll
          for (int ks = 0; ks < KSP; ++ks) {
            const int kk = 4 * ks + lc;
            afr[mt][ks] = (TBW && kk < P) ? (ptab == 0 ? sB : sG)[(8 * mt + lr) * P + kk] : 0.0;
          }
#pragma unroll
        for (int rr = 0; rr < (NTILE + NTH / 32 - 1) / (NTH / 32); ++rr) {
          const int tl = !TBW ? warp + rr * (NTH / 32)
                              : (warp < 5 ? (warp + 5 * rr < NB ? warp + 5 * rr : NTILE) : NB + (warp - 5) + 3 * rr);
          if (tl < NTILE) {
            const int tab = tl < NB ? 0 : tl < NB + NG ? 1 : 2;      // 0: B, 1: G, 2: Phi (warp-uniform)
            const int c0 = (tab == 0 ? tl : tab == 1 ? tl - NB : 0) * 8;
            const double *X = tab == 0 ? sB : tab == 1 ? sG : sPhi;
            const int ldx = tab == 2 ? Dm::TS : P, kx = tab == 2 ? T : P, ncol = tab == 0 ? 108 : tab == 1 ? 54 : T;
            // B operand In[a1][col]: the [a1][108] T lines (B and G tables) or TE[j1][j0] (Phi): linear in col
            const int bcol = c0 + lr;
            const double *bsrc = (tab == 2 ? sA + 12 * P2 : sA) + bcol;
            const int bstride = tab == 2 ? T : 108;
            const bool bok = bcol < ncol;
            double d[2][2] = {{0.0, 0.0}, {0.0, 0.0}};
#pragma unroll
            for (int ks = 0; ks < KSP; ++ks) {
              const int kk = 4 * ks + lc;
              if (tab != 2 || ks < KST) {
                const double b = (bok && kk < kx) ? bsrc[kk * bstride] : 0.0;
#pragma unroll
                for (int mt = 0; mt < 2; ++mt) {
                  const double af = (TBW && tab == ptab) ? afr[mt][ks] : (kk < kx ? X[(8 * mt + lr) * ldx + kk] : 0.0);
                  dmma(d[mt][0], d[mt][1], af, b);
                }
              }
            }
#pragma unroll
            for (int i = 0; i < 2; ++i) {
              const int col = c0 + 2 * lc + i;
              if (col < ncol) {
                double *dst;
                bool pad = false;
                if (tab == 2) {
                  dst = sBr + 18 * N * PP + lr * T + col;
                } else {
                  const int fa = (col * 57) >> 9;   // = col / 9 for col < 108
                  const int a0 = col - fa * P;
                  const int fm = tab == 1 ? 3 * fa + 1 : (fa < 6 ? 3 * fa : 3 * (fa - 6) + 2);
                  dst = sBr + fm * N * PP + lr * PP + a0;
                  pad = P < PP && a0 == P - 1;
                }
                const int mstride = tab == 2 ? 8 * T : 8 * PP;   // m-tile 1 = q1 + 8
#pragma unroll
                for (int mt = 0; mt < 2; ++mt) {
                  dst[mt * mstride] = d[mt][i];
                  if (pad) dst[mt * mstride + 1] = 0.0;   // zero pad of the 16-byte pairs
                }
              }
            }
          }
        }
      } else {
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
      // ---- stage C (a0 -> q0) + point evaluation ----------------------------------------------------
      double dslab = __longlong_as_double(0x7ff0000000000000LL);   // SDT: this thread's dt of the slab (0: det J <= 0)
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
          point_eval3<true, 0, (MB & 128) ? 6 : 0>(Jm, Gv, eq, R, alpha, sJ0[9], sJ0, a.ph, pt, best);
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
        if (SDT) {
          dslab = pt.bad ? 0.0 : pt.dt;
        } else {
          dtmin = fmin(dtmin, pt.dt);
          bad |= pt.bad;
        }
      }
      if (SDT) {   // dt >= 0: doubles order like their bit patterns, so an integer min is the min
#pragma unroll
        for (int sft = 16; sft > 0; sft >>= 1) dslab = fmin(dslab, __shfl_xor_sync(0xffffffffu, dslab, sft));
        if (lane == 0)
          atomicMin(reinterpret_cast<unsigned long long *>(sRed + 10), (unsigned long long)__double_as_longlong(dslab));
      }
      __syncthreads();
      // ---- stage C^T: q0 -> a0; warps 0-1: d = 0 components (G), 2-4: d != 0 (B), 5: Pq (Phi) -------
      if (MB & 4) {
        // DMMA form (MB bit 2): Y[cd][q1][a0] = sum_q0 X(q0, a0) S[cd][q1][q0] with M = a0 0..7 (one tile),
        // K = q0 (four steps), N = q1 (two tiles); X = G for d = 0, B otherwise, Phi for the Pq lines (cd = 9,
        // M = j0).  20 units (cd, q1 tile) over the 8 warps; the a0 = P-1 = 8 row by DFMA on threads 112-255.
        static_assert(!(MB & 4) || (N == 16 && P == 9 && T == 8), "DMMA stage C^T is written for k = 8");
        const int lr = lane >> 2, lc = lane & 3;
#pragma unroll 1
        for (int rr = 0; rr < 3; ++rr) {
          const int u = warp + 8 * rr;
          if (u < 20) {
            const int cd = u >> 1, nt = u & 1;
            const double *X = cd == 9 ? sPhi : (cd % 3 == 0 ? sG : sB);
            const int ldx = cd == 9 ? Dm::TS : P;
            const double *Sb = sA + (cd * N + 8 * nt + lr) * SR;   // B[q0][q1 = lr] = S[cd][q1][q0]
            double d0 = 0.0, d1 = 0.0;
#pragma unroll
            for (int ks = 0; ks < 4; ++ks) {
              const int qq0 = 4 * ks + lc;
              dmma(d0, d1, X[qq0 * ldx + lr], Sb[qq0]);           // A[a0 = lr][q0 = lc]
            }
            const int qa = 8 * nt + 2 * lc;
            if (cd < 9) {
              sBr[(cd * N + qa) * P + lr] = d0;
              sBr[(cd * N + qa + 1) * P + lr] = d1;
            } else {
              sBr[9 * N * P + lr * N + qa] = d0;
              sBr[9 * N * P + lr * N + qa + 1] = d1;
            }
          }
        }
        if (tid >= NTH - 9 * N) {   // the a0 = 8 row: 144 rows (cd, q1), 16 DFMA each
          const int it = tid - (NTH - 9 * N), cd = it / N, qq1 = it - cd * N;
          const double *X = cd % 3 == 0 ? sG : sB;
          const double *row = sA + (cd * N + qq1) * SR;
          double y = 0.0;
#pragma unroll
          for (int qq0 = 0; qq0 < N; ++qq0) y = fma(X[qq0 * P + P - 1], row[qq0], y);
          sBr[(cd * N + qq1) * P + P - 1] = y;
        }
      } else {
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
      // ---- stage B^T: q1 -> a1 on all 8 warps: warps 0..NPART-1 ZB items (c, a0) for a1 part = warp,
      //      the next NPART warps ZG items, the rest ZE items (j0) for j1 halves ------------------------
      if (MB & 2) {
        // DMMA form (MB bit 1): ZB[c][a1][a0] = sum_q1 B(q1,a1) Y0[c][q1][a0] + G(q1,a1) Y1[c][q1][a0] and
        // ZG[c][a1][a0] = sum_q1 B(q1,a1) Y2[c][q1][a0] with M = a1 0..7 (one tile), K = q1 (four steps),
        // N = (c, a0) columns 9 c + a0 (four tiles, warps 0-3); ZE[j1][j0] = sum_q1 Phi(q1,j1) YE[j0][q1] on
        // warp 4; the a1 = P-1 = 8 row of ZB / ZG by DFMA on warp 5.
        static_assert(!(MB & 2) || (N == 16 && P == 9 && T == 8), "DMMA stage B^T is written for k = 8");
        const int lr = lane >> 2, lc = lane & 3;
        if (warp < 4) {
          const int bcol = 8 * warp + lr;                       // this lane's B-operand column (c, a0)
          const bool bok = bcol < 27;
          const int bc = (bcol * 57) >> 9, ba0 = bcol - 9 * bc;  // / 9 and % 9 for bcol < 108
          const double *y0 = sBr + (3 * bc) * N * P + ba0, *y1 = y0 + N * P, *y2 = y0 + 2 * N * P;
          double zb0 = 0.0, zb1 = 0.0, zg0 = 0.0, zg1 = 0.0;
#pragma unroll
          for (int ks = 0; ks < 4; ++ks) {
            const int qq1 = 4 * ks + lc;
            const double aB = sB[qq1 * P + lr], aG = sG[qq1 * P + lr];    // A[a1 = lr][q1 = lc]
            const double b0 = bok ? y0[qq1 * P] : 0.0, b1 = bok ? y1[qq1 * P] : 0.0, b2 = bok ? y2[qq1 * P] : 0.0;
            dmma(zb0, zb1, aB, b0);
            dmma(zb0, zb1, aG, b1);
            dmma(zg0, zg1, aB, b2);
          }
#pragma unroll
          for (int i = 0; i < 2; ++i) {
            const int col = 8 * warp + 2 * lc + i;
            if (col < 27) {
              const int c = (col * 57) >> 9, a0 = col - 9 * c;
              sA[c * P2 + lr * P + a0] = i ? zb1 : zb0;
              sA[3 * P2 + c * P2 + lr * P + a0] = i ? zg1 : zg0;
            }
          }
        } else if (warp == 4) {
          double e0 = 0.0, e1 = 0.0;
#pragma unroll
          for (int ks = 0; ks < 4; ++ks) {
            const int qq1 = 4 * ks + lc;
            dmma(e0, e1, sPhi[qq1 * Dm::TS + lr], sBr[9 * N * P + lr * N + qq1]);   // A[j1][q1], B[q1][j0 = lr]
          }
          sA[6 * P2 + lr * T + 2 * lc] = e0;
          sA[6 * P2 + lr * T + 2 * lc + 1] = e1;
        } else if (warp == 5 && lane < 27) {
          const int c = (lane * 57) >> 9, a0 = lane - 9 * c;
          const double *y0 = sBr + (3 * c) * N * P + a0, *y1 = y0 + N * P, *y2 = y0 + 2 * N * P;
          double sb = 0.0, sg = 0.0;
#pragma unroll
          for (int qq1 = 0; qq1 < N; ++qq1) {
            const double bq = sB[qq1 * P + P - 1], gq = sG[qq1 * P + P - 1];
            sb = fma(bq, y0[qq1 * P], sb);
            sb = fma(gq, y1[qq1 * P], sb);
            sg = fma(bq, y2[qq1 * P], sg);
          }
          sA[c * P2 + (P - 1) * P + a0] = sb;
          sA[3 * P2 + c * P2 + (P - 1) * P + a0] = sg;
        }
      } else {
        const CTZ<K> C{4 * o};
        if (warp < NPART) {
          if (lane < 3 * P) {
            const int c = lane / P, a0 = lane - c * P, p0 = warp * PL;
            const double *y0 = sBr + ((c * 3 + 0) * N) * P + a0, *y1 = sBr + ((c * 3 + 1) * N) * P + a0;
            double v0[N], v1[N];
#pragma unroll
            for (int qq1 = 0; qq1 < N; ++qq1) { v0[qq1] = y0[qq1 * P]; v1[qq1] = y1[qq1 * P]; }
#pragma unroll
            for (int k1 = 0; k1 < PL; ++k1) {
              double s = 0.0;
#pragma unroll
              for (int qq1 = 0; qq1 < N; ++qq1) {
                s = fma(C.B(qq1, p0 + k1), v0[qq1], s);
                s = fma(C.G(qq1, p0 + k1), v1[qq1], s);
              }
              sA[c * P2 + (p0 + k1) * P + a0] = s;
            }
          }
        } else if (warp < 2 * NPART) {
          if (lane < 3 * P) {
            const int c = lane / P, a0 = lane - c * P, p0 = (warp - NPART) * PL;
            const double *y2 = sBr + ((c * 3 + 2) * N) * P + a0;
            double v2[N];
#pragma unroll
            for (int qq1 = 0; qq1 < N; ++qq1) v2[qq1] = y2[qq1 * P];
#pragma unroll
            for (int k1 = 0; k1 < PL; ++k1) {
              double s = 0.0;
#pragma unroll
              for (int qq1 = 0; qq1 < N; ++qq1) s = fma(C.B(qq1, p0 + k1), v2[qq1], s);
              sA[3 * P2 + c * P2 + (p0 + k1) * P + a0] = s;
            }
          }
        } else {
          constexpr int NEW = NTH / 32 - 2 * NPART;   // warps for the ZE items
          constexpr int JL = (T + NEW - 1) / NEW;
          const int j10 = (warp - 2 * NPART) * JL;
          if (lane < T) {
            const int j0 = lane;
            double ve[N];
#pragma unroll
            for (int qq1 = 0; qq1 < N; ++qq1) ve[qq1] = sBr[9 * N * P + j0 * N + qq1];
#pragma unroll
            for (int k1 = 0; k1 < JL; ++k1) {
              if (j10 + k1 < T) {
                double s = 0.0;
#pragma unroll
                for (int qq1 = 0; qq1 < N; ++qq1) s = fma(C.Phi(qq1, j10 + k1), ve[qq1], s);
                sA[6 * P2 + (j10 + k1) * T + j0] = s;
              }
            }
          }
        }
      }
      __syncthreads();
      // ---- stage A^T: accumulate q2 -> a2; item (c, a1 a0) owns 9 accumulators, e items on the top -
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
    // ---- zone outputs; accumulators cleared for the next zone (same thread <-> entry mapping) -------
    for (int i = tid; i < 3 * NK; i += NTH) { a.Fz1[z * 3 * NK + i] = sAF[i]; sAF[i] = 0.0; }
    for (int i = tid; i < NT; i += NTH) { a.FTv[z * NT + i] = sAE[i]; sAE[i] = 0.0; }
    cp_async_wait<0>();   // the next zone's X, V, e, J0^{-1} (issued in the last slab)
    __syncthreads();
  }
  if (SDT) {   // the last __syncthreads of the zone loop ordered every warp's atomicMin before this read
    if (tid == 0) a.cta_dt[blockIdx.x] = nz > 0 ? sRed[10] : __longlong_as_double(0x7ff0000000000000LL);
    return;
  }
  if (bad) dtmin = 0.0;
  const double m = block_min(dtmin, sRed);
  if (tid == 0) a.cta_dt[blockIdx.x] = m;
}
