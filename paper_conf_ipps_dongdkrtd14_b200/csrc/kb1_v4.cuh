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

// (round 2) The kb1_v4_3d kernel itself — the first warp-specialized pipeline, superseded by v5 / v10 and no
// longer a candidate — was removed; its measurements are in DESIGN.md §10 and git history.  This header keeps
// the pieces its successors build on: V4Dims, KB1V4Cfg, opaque_tid, kw_bar, cta_bar_div.
