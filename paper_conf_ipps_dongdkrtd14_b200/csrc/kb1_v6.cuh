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

// (round 2) The kb1_v6_3d kernel itself (contraction warps all on DFMA; superseded by v10, which keeps its
// forward stages) was removed; its measurements are in DESIGN.md §10 and git history.  This header keeps
// js_idx, lds_f64x2 and CTZ, which v10 and v8 / v11 use.
