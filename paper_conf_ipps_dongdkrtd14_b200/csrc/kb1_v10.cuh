// KB1 v10 — warp-specialized 3D corner force (k = 4): v6's DFMA forward stages, v5's DMMA back stages.
//
// Same mathematics, buffers, point warps and swizzled J/S layout as kb1_v6.cuh (eq (4)-(6);
// DESIGN.md §1 rows a0-a5).  The stage clocks of the contraction warps alone (profiles/r01_kw_stage_clocks.txt)
// split the two choices by direction: the forward stages A, B, C_x cost about the same on DFMA (v6.d2:
// 1045 + 1615 + 1549 cycles per zone) as on DMMA (v5.d2: 1211 + 2086 + 1080), the back stages C^T, B^T, A^T
// are much cheaper on DMMA (1615 + 1428 + 845 vs 1955 + 2065 + 1420).  Every DMMA, on the other hand, blocks
// the point warps' DFMAs for 16 pipe cycles (profiles/r01_pipe_share.txt).  So the forward stages run on
// DFMA (no padding, 2-cycle pipe quanta) and only the back stages on DMMA: about 40 % of v5's DMMA pipe time.
// The back stages read S through the v6 pair swizzle (js_idx).
//
// OPT bit 0 (BULK): e and rho0|J0| of the next zone (contiguous, 512 + 4096 bytes) arrive by two
// cp.async.bulk copies issued by one thread and completed on an mbarrier, instead of 576 8-byte cp.asyncs
// spread over the contraction warps (their issue phase was 2.4 K cycles per zone next to the point warps).
// OPT bit 1 (LATE): the gather of zone i+1 is issued after the C^T stage of zone i-1 instead of before it,
// away from the point warps' stage-C shared-memory burst at the start of every zone.
// OPT bit 2 (BAL): forward stage B's 32 e items go two each to the 16 threads without a field item.
// OPT bit 4 (V16): e and rho0|J0| (contiguous per zone) by 16-byte cp.async.
// OPT bit 6 (SPREAD): the x / v node gather spread over all contraction threads (3 copies each).
// OPT bit 3 (PWG): the POINT warps issue the gather of zone i+2 at the end of their zone i (they finish
// before the contraction warps, which are the bound), into a second XE buffer; completion reaches the
// contraction warps through cp.async.mbarrier.arrive on a per-buffer mbarrier, so the contraction warps
// issue nothing (their issue phase was 2.2 K of 11.7 K cycles per zone next to the point warps).
#pragma once
#include "kb1_v6.cuh"

__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
                   smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void cp_async16(void *dst, const void *src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_mbar_arrive(uint64_t *bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, unsigned parity) {
  asm volatile(
      "{\n.reg .pred p;\nWAIT_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra WAIT_%=;\n}\n" ::"r"(
          smem_u32(bar)), "r"(parity)
      : "memory");
}

// OPT bit 7 (PADU): padded U layouts for the forward stage B stores.  With the natural layout
// U[cm][q2][q1][a0] (q2 stride N*P = 40) a half-warp of stage B (16 consecutive (q2, a0) items, one q1)
// touches only 10 distinct 8-byte banks (40 = 8 mod 16): 2-way conflicts on all 24 stores per item, and the
// e items' UE[q2][q1][j0] (q2 stride 32) are 4-way.  PADU uses q2 stride UQ = 53 (= 5 mod 16: a half-warp's
// 16 items land on 16 banks) and q1 stride UQ1 = 6 (keeps stage C's half-warps -- q2 pair x 8 q1 at fixed a0
// -- and the point warps' 8 q1 per warp conflict-free), and UE q2 stride N*T + 4 (bit 9, PADE, alone).
// Bank model: tools/v10_stageB_bank_model.py (stage B 784 -> 400 wavefronts per zone, stage C unchanged).
// Measured (profiles/r01_bench_c4_v10wu_*.jsonl): store conflicts 23.6 M -> 10.8 M per launch, but 2.7 %
// SLOWER: the extra 22.5 KB shrink L1 (228 KB - shared) from ~33 to ~10 KB, below the point warps' 30 KB
// spill working set, and the spill reloads miss (3.3 M -> 7.6 M local sectors).  v10.wpad (v10.w + the same 22.5 KB
// unused, OPT bit 10) is exactly as slow, so the conflicts themselves were off the critical path.
template <int K, bool PADU, bool PADE = PADU, bool XEB = true>
struct V10Dims : V5Dims<K> {
  using B = V5Dims<K>;
  using B::N, B::P, B::T, B::N2, B::N3, B::TAB, B::JSBUF, B::XE, B::P3, B::O_UX, B::YZREG;
  static_assert(!PADU || K == 4, "PADU strides are chosen for k = 4 (N = 8, P = 5)");
  static constexpr int UQ = PADU ? 53 : N * P, UQ1 = PADU ? 6 : P, UM = N * UQ, UQE = PADE ? N * T + 4 : N * T;
  static constexpr int O_UE = 9 * UM, O_R = (O_UE + N * UQE + 1) / 2 * 2, UVBUF = (O_R + N3 + 1) / 2 * 2;
  static constexpr int FWREG = O_UX + 9 * UM;
  static constexpr int WREG = ((FWREG > YZREG ? FWREG : YZREG) + 1) / 2 * 2;
  static constexpr int OFF_JS = TAB, OFF_UV = OFF_JS + 2 * JSBUF, OFF_XE = OFF_UV + 2 * UVBUF, OFF_W = OFF_XE + XE;
  static constexpr int OFF_J = OFF_W + WREG;
  static constexpr int OFF_RED = OFF_J + 20;
  static constexpr int OFF_ID = OFF_RED + 32;
  static constexpr int OFF_MB = OFF_ID + (2 * P3 + 1) / 2;
  static constexpr int OFF_XEB = OFF_MB + 2;
  static constexpr int TOTAL = OFF_XEB + (XEB ? XE : 0);   // the second XE buffer serves PWG only
};
template <int K, int OPT>
constexpr int v10_smem_bytes() {   // OPT bit 10: PADU's extra 2872 doubles, unused (diagnostic: the L1 share)
  return (V10Dims<K, (OPT & 128) != 0, (OPT & 640) != 0, (OPT & 8) || !(OPT & 2048)>::TOTAL + ((OPT & 1024) ? 2872 : 0)) * 8;
}

template <int K, int DIAG = 0, int MODE = 0, int OPT = 0, int VMODE_ = 0>
__global__ void __launch_bounds__(KB1V5Cfg<K, MODE>::NTH, 1) kb1_v10_3d(const KB1Args a) {
  using Dm = V10Dims<K, (OPT & 128) != 0, (OPT & 640) != 0, (OPT & 8) || !(OPT & 2048)>;   // bit 11: no XEB   // OPT bit 9 (PADE): the UE padding alone
  constexpr int UQ = Dm::UQ, UQ1 = Dm::UQ1, UM = Dm::UM, UQE = Dm::UQE;
  using Cfg = KB1V5Cfg<K, MODE>;
  constexpr bool BULK = OPT & 1, LATE = OPT & 2, BAL = OPT & 4, PWG = OPT & 8, V16 = OPT & 16;
  constexpr bool NOXV = OPT & 32;   // timing diagnostic only (wrong results): no x / v gather
  constexpr bool CLK = !(OPT & 4096);   // per-zone clock64 accounting (BLAST_CF_PROFILE); bit 12 compiles it out
  constexpr int EIG = (OPT & 8192) ? 1 : (OPT & 32768) ? 2 : (OPT & 524288) ? 3 : (OPT & 2097152) ? 4 : (OPT & (1 << 30)) ? 5 : (VMODE_ & 8) ? 6 : 0;   // bit 30: the shorter-chain eigenpair   // bit 19: diagnostic, no complement   // bits 13 / 15: branchy / warp-uniform shortcut of the eigenpair
  // bit 14 (RHOPW): rho0|J0| is not staged by the contraction warps (512 of their ~1340 cp.async per zone);
  // the point warps prefetch zone i+1's into L2 while they work on zone i and load their two values directly
  constexpr bool RHOPW = OPT & 16384;
  // bit 16 (EARLYS): each point's S, P go to the JS buffer right after its evaluation (its J is dead), and the
  // exact dt of the candidates comes from the J^T J the evaluation kept: point a's S is not live across point b
  constexpr bool EARLYS = OPT & 65536;
  // VMODE_ bits 0-1: the point evaluation's switch mode; bits 2+: more options (OPT's bits are used up)
  constexpr int VMODE = VMODE_ & 3;
  // VMODE_ bit 2 (DCT): stage C^T on DFMA (v6's form: one (row c, col) item per contraction thread, constant-bank
  // tables) instead of DMMA -- 2-cycle pipe quanta next to the point warps' DFMAs instead of 16-cycle DMMA tiles
  constexpr bool DCT = VMODE_ & 4;
  // VMODE_ bit 4 (KWB, needs PCT): the contraction warps compute every point's dt-filter bound (J^T J and
  // q - sqrt(2/3) |J^T J - q I|_F, pointwise.cuh dt_filter_bound_J) right after stage C_x, into the JS buffer's
  // tenth plane (free until the point warps' YE stores): ~30 FP64 instructions per point off the point warps
  constexpr bool KWB = VMODE_ & 16;
  constexpr bool SPREAD = OPT & 64;   // the 6 P^3 node-field copies spread over all contraction threads
  // bits 17 / 18 (timing diagnostics, wrong dt by design): the exact dt of FILTER 2 never / always evaluated
  // bit 25 (PCT): the POINT warps run the back stage C^T themselves, on DMMA straight from the S values in their
  // registers -- lane l's two points (q0 = l % 4 and l % 4 + 4, q1 = l / 4, q2 = warp) are exactly the B fragments
  // of the m8n8k4 tile (k = q0, n = q1) for k-steps 0 and 1 -- and store Y[cd][a0][q1] into their own warp's
  // rows of the JS buffer (rows col = 8 q2 .. 8 q2 + 7, which only this warp reads); S is never stored and the
  // contraction warps' back pass starts at B^T
  // bit 26 (PCTH): the point warps contract fields cd = 0..4 that way, the contraction warps the rest (5..9), also
  // writing Y into the JS rows (a warp's tile = one q2 row block, read and overwritten by that warp alone)
  constexpr int NPC = (OPT & (1 << 25)) ? 10 : (OPT & (1 << 26)) ? 5 : 0;   // fields the point warps contract
  constexpr bool PCT = NPC > 0;
  // bit 29 (FF, needs PCT): the contraction warps run zone i+1's forward stages A, B FIRST, then zone i-1's B^T,
  // then C_x(i+1) and A^T(i-1): no DMMA burst at the start of a period (where the point warps' stage C_v and J
  // loads are).  Z / ZE move below UX (over the dead T), the node gather runs two zones ahead into the two XE
  // buffers, rho0|J0| one zone ahead, and the contraction warps' cp.async wait moves to the end of the period.
  constexpr bool FF = OPT & (1 << 29);
  static_assert(!FF || (PCT && !PWG && !BULK && !LATE && !RHOPW && !SPREAD && !V16), "FF: PCT layout, plain gather");
  constexpr int O_Z = FF ? 0 : Dm::O_Z, O_ZE = FF ? 6 * Dm::N * Dm::P2 : Dm::O_ZE;
  static_assert(!FF || 6 * Dm::N * Dm::P2 + Dm::N * Dm::T2 <= Dm::O_UX, "FF: Z / ZE must stay below UX");
  constexpr unsigned KSLEEP = ((OPT >> 27) & 3) * 200;   // bits 27-28: timing experiment, contraction warps sleep 200-600 ns   // Y[cd][a0][col] lives in the JS buffer (plane cd, slot q2 * N^2 + a0 * N + q1)
  constexpr bool NOCV = OPT & 1048576;
  // bits 21-24 (timing diagnostics, wrong): skip the contraction stage C^T / B^T + A^T / forward A + B / forward C_x
  constexpr bool SKCT = OPT & (1 << 21), SKBA = OPT & (1 << 22), SKAB = OPT & (1 << 23), SKCX = OPT & (1 << 24);   // bit 20 (timing diagnostic, wrong): no stage C of the velocity fields
  constexpr int DTX = (OPT & 131072) ? 1 : (OPT & 262144) ? 2 : 0;
  static_assert(!V16 || (Dm::T3 % 2 == 0 && Dm::N3 % 2 == 0 && Dm::XE_E % 2 == 0 && (Dm::OFF_XE + Dm::XE_E) % 2 == 0 &&
                         (Dm::OFF_UV + Dm::O_R) % 2 == 0 && Dm::UVBUF % 2 == 0), "16-byte copies need 16-byte alignment");
  static_assert(!(PWG && (BULK || LATE)), "PWG replaces the contraction warps' gather");
  static_assert(!BULK || ((Dm::OFF_XE + Dm::XE_E) % 2 == 0 && (Dm::OFF_UV + Dm::O_R) % 2 == 0 && Dm::UVBUF % 2 == 0 &&
                          (Dm::T3 * 8) % 16 == 0 && (Dm::N3 * 8) % 16 == 0),
                "bulk copies need 16-byte aligned, 16-byte multiple destinations");
  constexpr int N = Dm::N, P = Dm::P, T = Dm::T, P2 = Dm::P2, P3 = Dm::P3, T2 = Dm::T2, T3 = Dm::T3;
  constexpr int N2 = Dm::N2, N3 = Dm::N3, NH = Dm::NH, TPZ = Dm::TPZ;
  constexpr int NPW = Cfg::NPW, NKW = Cfg::NKW, NKWW = NKW / 32, KWCH = Cfg::KWCH;
  constexpr int KS_N = Dm::KS_N;
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
  // VMODE_ bit 5 (NOKST): the contraction warps' per-stage clock stamps compiled out (each is a runtime-checked
  // branch at a stage barrier; the per-zone accounting of CLK stays)
  constexpr bool KST = !(VMODE_ & 32);
  // VMODE_ bits 6 / 7 (PFENCE, experiment): runtime-uniform, never-taken branches in the point warps' zone body
  // (after stage C_v / before the C^T tiles) -- the contraction warps' stage stamps turned out to be scheduling
  // fences ptxas benefits from (compiling them out: 11 % slower)
  constexpr int PFENCE = (VMODE_ >> 6) & 3;
  // VMODE_ bits 8 / 9 (KFENCE, experiment): a never-taken stamp branch between the work blocks of the forward
  // stages A, B (bit 8) and C_x (bit 9), so ptxas does not interleave the blocks' loads
  constexpr int KFENCE = (VMODE_ >> 8) & 3;
  // VMODE_ bit 10 (FBM): forward stage B on DMMA instead of DFMA + LDCU (the C5 lesson)
  constexpr bool FBM = VMODE_ & 1024;
  constexpr bool PADU_ = (OPT & 128) != 0;
  auto pfence = [&](int slot) {
    if (a.prof != nullptr && tid == 0) sKP[12 + slot] = clock64();
  };
  auto kstamp = [&](int slot) {
    if (KST && a.prof != nullptr && tid == NPW) {
      const long long t = clock64();
      sKP[slot] += t - sKP[15];
      sKP[15] = t;
    }
  };

  for (int i = tid; i < 2 * N * P + N * T + N; i += Cfg::NTH) sTab[i] = __ldg(a.tab + i);
  if (tid == 0) sRed[8] = 0.0;   // dt filter: best exact inverse dt of this CTA (point_eval3<true>)

  double *const sXEb[2] = {sXE, smem + Dm::OFF_XEB};   // PWG: XE of zone i is sXEb[i & 1]
  if (PWG) {
    if (tid == 0) {
      mbar_init(reinterpret_cast<uint64_t *>(smem + Dm::OFF_MB), NPW);
      mbar_init(reinterpret_cast<uint64_t *>(smem + Dm::OFF_MB) + 1, NPW);
      asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    __syncthreads();
  }
  // ---------------- KW ----------------
  // node ids travel by cp.async into shared memory one zone ahead (a register copy of an __ldg result
  // would be spilled by the 88-register warps and the spill store would wait for the load)
  int32_t *sID = reinterpret_cast<int32_t *>(smem + Dm::OFF_ID);
  uint64_t *sMB = reinterpret_cast<uint64_t *>(smem + Dm::OFF_MB);
  auto kw_load_id = [&](int64_t i) {
    if (i < nz && ktid < P3) cp_async4(sID + (i & 1) * P3 + ktid, a.zone_nodes + zone_of(i) * P3 + ktid);
  };
  auto kw_issue = [&](int64_t i) {       // cp.async gather of zone i into XE and R of UV[i & 1]
    if (i < nz) {
      const int64_t z = zone_of(i);
      if (SPREAD) {   // item (f, a): warps 0-7 each take ~3 copies instead of warps 0-3 taking 6
        for (int it2 = ktid; it2 < 6 * P3; it2 += NKW) {
          const int f = it2 / P3, aa = it2 - f * P3;
          const int64_t node = sID[(i & 1) * P3 + aa];
          cp_async8(sXE + Dm::XE_X + f * P3 + aa, (f < 3 ? a.x + f * nn : a.v + (f - 3) * nn) + node, true);
        }
      } else if (!NOXV && ktid < P3) {
        const int64_t node = sID[(i & 1) * P3 + ktid];
#pragma unroll
        for (int c = 0; c < 3; ++c) {
          cp_async8(sXE + Dm::XE_X + c * P3 + ktid, a.x + c * nn + node, true);
          cp_async8(sXE + Dm::XE_X + (3 + c) * P3 + ktid, a.v + c * nn + node, true);
        }
      }
      double *R = sUV + (i & 1) * Dm::UVBUF + Dm::O_R;
      if (RHOPW) {
        for (int r = ktid; r < T3 + 10; r += NKW) {
          const double *src = r < T3 ? a.e + z * T3 + r : r < T3 + 9 ? a.J0inv + z * 9 + (r - T3) : a.zone_gamma + z;
          cp_async8(sXE + Dm::XE_E + r, src, true);
        }
      } else if (BULK) {
        if (ktid == 0) {
          uint64_t *bar = sMB + (i & 1);
          mbar_expect_tx(bar, (T3 + N3) * 8);
          bulk_g2s(sXE + Dm::XE_E, a.e + z * T3, T3 * 8, bar);
          bulk_g2s(R, a.rho0detJ0 + z * N3, N3 * 8, bar);
        }
        if (ktid < 10) cp_async8(sXE + Dm::XE_J + ktid, ktid < 9 ? a.J0inv + z * 9 + ktid : a.zone_gamma + z, true);
      } else if (V16) {   // e and rho0|J0| are contiguous per zone: 16-byte copies, half the instructions
        for (int r = 2 * ktid; r < T3; r += 2 * NKW) cp_async16(sXE + Dm::XE_E + r, a.e + z * T3 + r);
        if (ktid < 10) cp_async8(sXE + Dm::XE_J + ktid, ktid < 9 ? a.J0inv + z * 9 + ktid : a.zone_gamma + z, true);
        for (int r = 2 * ktid; r < N3; r += 2 * NKW) cp_async16(R + r, a.rho0detJ0 + z * N3 + r);
      } else {
        for (int r = ktid; r < T3 + 10; r += NKW) {
          const double *src = r < T3 ? a.e + z * T3 + r : r < T3 + 9 ? a.J0inv + z * 9 + (r - T3) : a.zone_gamma + z;
          cp_async8(sXE + Dm::XE_E + r, src, true);
        }
        for (int r = ktid; r < N3; r += NKW) cp_async8(R + r, a.rho0detJ0 + z * N3 + r, true);
      }
    }
  };
  // the bulk copies of zone i have landed (every contraction thread waits; phase = use count of the buffer)
  auto kw_wait_bulk = [&](int64_t i) {
    if (BULK && i < nz) mbar_wait(sMB + (i & 1), (unsigned)((i >> 1) & 1));
  };
  // part: 0 = stages A, B, C_x; 1 = A, B only; 2 = C_x only (FF)
  auto kw_forward = [&](double *ub, double *jb, double *js, int zc, const double *xe, int part = 0) {
    const int kt = opaque_tid() - NPW;
    double *Tr = sWk, *UX = sWk + Dm::O_UX;
    if (part != 2) {
    if (kt < 10) js[kt] = xe[Dm::XE_J + kt];
    // stage A: a2 -> q2 (T_B, T_G of the 6 fields; TE of e)
    {
    const int r0_ = kt;
#pragma unroll
    for (int blk = 0; blk < (SKAB ? 0 : (6 * P2 + T2 + NKW - 1) / NKW); ++blk) {
      const int r = r0_ + blk * NKW;
      if ((KFENCE & 1) && blk > 0) kstamp(14);
      const CTZ<K> C{zc * (blk + 1)};
      if (r < 6 * P2 + T2) {
      if (r < 6 * P2) {
        const int f = r / P2, aa = r - f * P2;
        double xv[P];
#pragma unroll
        for (int a2 = 0; a2 < P; ++a2) xv[a2] = xe[Dm::XE_X + f * P3 + a2 * P2 + aa];
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
        for (int j2 = 0; j2 < T; ++j2) ev[j2] = xe[Dm::XE_E + j2 * T2 + jj];
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
    // (BAL: the second block's e items go to the threads without a field item, not to threads 0-15 again)
    if (FBM) {   // VMODE_ bit 10: stage B on DMMA (kb1_v5.cuh's form): M = q1, K = a1 (P padded to 8), N = (f, q2, a0)
      static_assert(!FBM || (!PADU_ && N == 8), "FBM: the natural U layout, one m-tile of q1");
      const int kt = opaque_tid() - NPW, kwarp = kt >> 5, lr = (kt & 31) >> 2, lc = kt & 3;
      constexpr int KS_P = (P + 3) / 4, KS_T = (T + 3) / 4;
      double fB[KS_P], fG[KS_P], fP[KS_T];
#pragma unroll
      for (int s2 = 0; s2 < KS_P; ++s2) {
        fB[s2] = tfrag<false>(tB, P, N, P, lr, 4 * s2 + lc);
        fG[s2] = tfrag<false>(tG, P, N, P, lr, 4 * s2 + lc);
      }
#pragma unroll
      for (int s2 = 0; s2 < KS_T; ++s2) fP[s2] = tfrag<false>(tPhi, T, N, T, lr, 4 * s2 + lc);
      constexpr int NC = 6 * N * P, NTL = (NC + 7) / 8, JPWT = (NTL + NKWW - 1) / NKWW;
#pragma unroll
      for (int t = 0; t < JPWT; ++t) {
        const int j = kwarp + t * NKWW;
        const int nb = min(j * 8 + lr, NC - 1);
        const int fb = nb / (N * P), rb = nb - fb * (N * P), q2b = rb / P, a0b = rb - q2b * P;
        const double *TBb = Tr + Dm::O_T + ((fb * 2 + 0) * N + q2b) * P2 + a0b;
        double u[3][2] = {{0.0, 0.0}, {0.0, 0.0}, {0.0, 0.0}};
#pragma unroll
        for (int s2 = 0; s2 < KS_P; ++s2) {
          const int a1 = min(4 * s2 + lc, P - 1);
          const double tb = TBb[a1 * P], tg = TBb[N * P2 + a1 * P];
          dmma(u[0][0], u[0][1], fB[s2], tb);
          dmma(u[1][0], u[1][1], fG[s2], tb);
          dmma(u[2][0], u[2][1], fB[s2], tg);
        }
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = j * 8 + 2 * lc + i;
          if (j < NTL && n < NC) {
            const int f = n / (N * P), rr = n - f * (N * P), q2 = rr / P, a0 = rr - q2 * P;
            double *U = (f < 3 ? UX + f * 3 * UM : ub + (f - 3) * 3 * UM) + q2 * UQ + lr * UQ1 + a0;
            U[0] = u[0][i];
            U[UM] = u[1][i];
            U[2 * UM] = u[2][i];
          }
        }
      }
      constexpr int NCE = N * T, NTE = (NCE + 7) / 8;   // UE = Phi . TE
      for (int te = kwarp; te < NTE; te += NKWW) {
        const int nb = min(te * 8 + lr, NCE - 1);
        const int q2b = nb / T, j0b = nb - q2b * T;
        double d0 = 0.0, d1 = 0.0;
#pragma unroll
        for (int s2 = 0; s2 < KS_T; ++s2) dmma(d0, d1, fP[s2], Tr[Dm::O_TE + q2b * T2 + min(4 * s2 + lc, T - 1) * T + j0b]);
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = te * 8 + 2 * lc + i;
          if (n < NCE) {
            const int q2 = n / T, j0 = n - q2 * T;
            ub[Dm::O_UE + q2 * UQE + lr * T + j0] = i ? d1 : d0;
          }
        }
      }
    } else
    {
    const int r0_ = opaque_tid() - NPW;
    constexpr int NB = 6 * N * P, NU = N * T;
    constexpr bool bal = BAL && NKW > NB && NU <= 2 * (NKW - NB) && (NB + NU + NKW - 1) / NKW == 2;
#pragma unroll
    for (int blk = 0; blk < (SKAB ? 0 : (6 * N * P + N * T + NKW - 1) / NKW); ++blk) {
      const int r = (bal && blk == 1) ? (r0_ >= NB ? NKW + r0_ - NB : NB + NU) : r0_ + blk * NKW;
      if ((KFENCE & 1) && blk > 0) kstamp(14);
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
        double *U0 = (f < 3 ? UX + f * 3 * UM : ub + (f - 3) * 3 * UM) + q2 * UQ + a0;
#pragma unroll
        for (int q1 = 0; q1 < N; ++q1) {
          double u0 = 0.0, u1 = 0.0, u2 = 0.0;
#pragma unroll
          for (int a1 = 0; a1 < P; ++a1) {
            u0 = fma(C.B(q1, a1), tb[a1], u0);
            u1 = fma(C.G(q1, a1), tb[a1], u1);
            u2 = fma(C.B(q1, a1), tg[a1], u2);
          }
          U0[q1 * UQ1] = u0;
          U0[UM + q1 * UQ1] = u1;
          U0[2 * UM + q1 * UQ1] = u2;
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
          ub[Dm::O_UE + q2 * UQE + q1 * T + j0] = ue;
        }
      }
    }}}
    kw_bar<NKW>();
    kstamp(9);
    }
    if (part == 1) return;
    // stage C (position fields): J[c][m](col, q0) = sum_a0 M_m[q0][a0] UX[c][m][col][a0] -> JS (swizzled)
    {
    const int r0_ = opaque_tid() - NPW;
#pragma unroll
    for (int blk = 0; blk < (SKCX ? 0 : (9 * N2 + NKW - 1) / NKW); ++blk) {
      const int r = r0_ + blk * NKW;
      if ((KFENCE & 2) && blk > 0) kstamp(14);
      const CTZ<K> C{zc * (blk + 1)};
      if (r < 9 * N2) {
      const int cm = r / N2, col = r - cm * N2;   // cm is warp-uniform (N2 = 64)
      double uv[P];
#pragma unroll
      for (int a0 = 0; a0 < P; ++a0) uv[a0] = UX[cm * UM + (col / N) * UQ + (col % N) * UQ1 + a0];
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
    if (KWB) {   // the dt-filter bound of every point of this zone into plane 9 (after all of J is stored)
      static_assert(!KWB || (PCT && N3 == 2 * NKW), "KWB: two points per contraction thread, plane 9 free (PCT)");
      kw_bar<NKW>();
      const int kt2 = opaque_tid() - NPW;
#pragma unroll 1
      for (int h = 0; h < 2; ++h) {
        const int pidx = kt2 + h * NKW, slot = js_idx(pidx >> 3, pidx & 7);
        double Jr[3][3];
#pragma unroll
        for (int cd = 0; cd < 9; ++cd) Jr[cd / 3][cd % 3] = jb[cd * N3 + slot];
        jb[Dm::O_PQ + slot] = dt_filter_bound_J(Jr);
      }
    }
    kstamp(10);
  };
  // back stages C^T, B^T, A^T of zone z from the JS buffer sb (S[9][N^3], Pq[N^3])
  // part: 0 = all back stages; 1 = C^T, B^T; 2 = A^T only (FF)
  auto kw_back = [&](const double *sb, int64_t z, int zc, auto &&mid, int part = 0) {
    const int ktid = opaque_tid() - NPW, kwarp = ktid >> 5, lr = (ktid & 31) >> 2, lc = ktid & 3;
    double fBt[KS_N], fGt[KS_N], fPt[KS_N];
#pragma unroll
    for (int s = 0; s < KS_N; ++s) {
      fBt[s] = tfrag<true>(tB, P, N, P, lr, 4 * s + lc);
      fGt[s] = tfrag<true>(tG, P, N, P, lr, 4 * s + lc);
      fPt[s] = tfrag<true>(tPhi, T, N, T, lr, 4 * s + lc);
    }
    double *Wr = sWk;
    if (part != 2) {
    if (DCT) {   // C^T on DFMA: q0 -> a0 for the 9 S components (3 items per col) and Pq
      static_assert(!DCT || NPC == 0, "DCT: S in the JS buffer");
      const int r = opaque_tid() - NPW;
      const CTZ<K> C{zc};
      if (r < 4 * N2) {
        const int c = r / N2, col = r - c * N2;   // warp-uniform c
        if (c < 3) {
#pragma unroll
          for (int d = 0; d < 3; ++d) {   // one S component at a time (register budget of the contraction warps)
            double sv[N];
            const double *bd = sb + (c * 3 + d) * N3;
#pragma unroll
            for (int pq = 0; pq < N / 2; ++pq) lds_f64x2(bd + js_idx(col, 2 * pq), sv[2 * pq], sv[2 * pq + 1]);
#pragma unroll
            for (int a0 = 0; a0 < P; ++a0) {
              double yv = 0.0;
#pragma unroll
              for (int q0 = 0; q0 < N; ++q0) yv = fma(d == 0 ? C.G(q0, a0) : C.B(q0, a0), sv[q0], yv);
              Wr[Dm::O_Y + ((c * 3 + d) * P + a0) * Dm::YS + col] = yv;
            }
          }
        } else {
          double pv[N];
#pragma unroll
          for (int pq = 0; pq < N / 2; ++pq) lds_f64x2(sb + Dm::O_PQ + js_idx(col, 2 * pq), pv[2 * pq], pv[2 * pq + 1]);
#pragma unroll
          for (int j0 = 0; j0 < T; ++j0) {
            double yv = 0.0;
#pragma unroll
            for (int q0 = 0; q0 < N; ++q0) yv = fma(C.Phi(q0, j0), pv[q0], yv);
            Wr[Dm::O_YE + j0 * Dm::YS + col] = yv;
          }
        }
      }
    } else
    if (NPC < 10) {   // C^T: each warp takes one column tile (col = q2*N + q1), five matrices at a time
      constexpr int NTL = (N2 + 7) / 8;
      for (int tl = kwarp; tl < (SKCT ? 0 : NTL); tl += NKWW) {
        const int colb = min(tl * 8 + lr, N2 - 1);
        int soff[KS_N];   // swizzled slot of this lane's q0 = 4 s + lc in row colb (kb1_v6.cuh js_idx), once per tile
#pragma unroll
        for (int s = 0; s < KS_N; ++s) soff[s] = js_idx(colb, min(4 * s + lc, N - 1));
#pragma unroll
        for (int h = NPC / 5; h < 2; ++h) {
          double sv[5][KS_N];
#pragma unroll
          for (int c5 = 0; c5 < 5; ++c5)
#pragma unroll
            for (int s = 0; s < KS_N; ++s) sv[c5][s] = sb[(h * 5 + c5) * N3 + soff[s]];
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
                if (PCT) {   // in place over this warp's own S rows (all its loads precede the DMMAs)
                  if (lr < (cd == 9 ? T : P)) const_cast<double *>(sb)[cd * N3 + tl * N2 + lr * N + 2 * lc + i] = d[c5][i];
                } else {
                if (cd < 9 && lr < P) Wr[Dm::O_Y + (cd * P + lr) * Dm::YS + col] = d[c5][i];
                if (cd == 9 && lr < T) Wr[Dm::O_YE + lr * Dm::YS + col] = d[c5][i];
                }
              }
            }
          }
        }
      }
    }
    if (NPC < 10) kw_bar<NKW>();
    kstamp(4);
    mid();
    {   // B^T
      constexpr int NC = N * P, NTL = (NC + 7) / 8, NJ = 3 * NTL, JPWT = (NJ + NKWW - 1) / NKWW, JPW = JPWT < KWCH ? JPWT : KWCH;
      for (int t0 = 0; t0 < (SKBA ? 0 : JPWT); t0 += JPW) {
        double y[JPW][3][KS_N];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = min(kwarp + (t0 + t) * NKWW, NJ - 1);
          const int c = j / NTL, tl = j - c * NTL;
          const int nb = min(tl * 8 + lr, NC - 1);
          const int q2b = nb / P, a0b = nb - q2b * P;
          if (PCT) {   // Y[cd][a0][q1] of column block q2 at JS plane cd, row block q2, slot a0 * 8 + q1
            const double *Yb = sb + (c * 3) * N3 + q2b * N2 + a0b * N;
#pragma unroll
            for (int s = 0; s < KS_N; ++s) {
              const int q1 = min(4 * s + lc, N - 1);
              y[t][0][s] = Yb[q1];
              y[t][1][s] = Yb[N3 + q1];
              y[t][2][s] = Yb[2 * N3 + q1];
            }
          } else {
          const double *Yb = Wr + Dm::O_Y + (c * 3 * P + a0b) * Dm::YS + q2b * N;
#pragma unroll
          for (int s = 0; s < KS_N; ++s) {
            const int q1 = min(4 * s + lc, N - 1);
            y[t][0][s] = Yb[q1];
            y[t][1][s] = Yb[P * Dm::YS + q1];
            y[t][2][s] = Yb[2 * P * Dm::YS + q1];
          }
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
              Wr[O_Z + ((c * 2 + 0) * N + q2) * P2 + lr * P + a0] = zb[t][i];
              Wr[O_Z + ((c * 2 + 1) * N + q2) * P2 + lr * P + a0] = zg[t][i];
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
        for (int s = 0; s < KS_N; ++s)
          dmma(d0, d1, fPt[s], PCT ? sb[9 * N3 + q2b * N2 + j0b * N + min(4 * s + lc, N - 1)]
                                   : Wr[Dm::O_YE + j0b * Dm::YS + q2b * N + min(4 * s + lc, N - 1)]);
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int n = te * 8 + 2 * lc + i;
          if (lr < T && n < NCE) {
            const int q2 = n / T, j0 = n - q2 * T;
            Wr[O_ZE + q2 * T2 + lr * T + j0] = i ? d1 : d0;
          }
        }
      }
    }
    kw_bar<NKW>();
    kstamp(5);
    }
    if (part == 1) return;
    {   // A^T -> global F_z.1 (zone-local) and F^T v
      constexpr int NTL = (P2 + 7) / 8, NJ = 3 * NTL, JPWT = (NJ + NKWW - 1) / NKWW, JPW = JPWT < KWCH ? JPWT : KWCH;
      for (int t0 = 0; t0 < (SKBA ? 0 : JPWT); t0 += JPW) {
        double zv[JPW][2][KS_N];
#pragma unroll
        for (int t = 0; t < JPW; ++t) {
          const int j = min(kwarp + (t0 + t) * NKWW, NJ - 1);
          const int c = j / NTL, tl = j - c * NTL;
          const int nb = min(tl * 8 + lr, P2 - 1);
          const double *Zb = Wr + O_Z + c * 2 * N * P2 + nb;
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
        for (int s = 0; s < KS_N; ++s) dmma(d0, d1, fPt[s], Wr[O_ZE + min(4 * s + lc, N - 1) * T2 + nb]);
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

  // ---------------- PW ----------------
  double dtmin = __longlong_as_double(0x7ff0000000000000LL);
  bool bad = false;
  long long nvote4 = 0, nexact4 = 0;   // DIAG 4 counters
  const int pr = tid, q0a = pr % NH, q1 = (pr / NH) % N, q2 = pr / (NH * N);
  auto pw_point = [&](const double *ub, const double *js, double *jb, int64_t z) {
    const double gamma = js[9];
    const int col = q2 * N + q1;
    const int qa = col * N + q0a, qb = qa + NH;                     // natural point index (R, Sq)
    const int sa = js_idx(col, q0a), sbi = js_idx(col, q0a + NH);  // JS slots
    const double Ra = RHOPW ? __ldg(a.rho0detJ0 + z * N3 + qa) : ub[Dm::O_R + qa];
    const double Rb = RHOPW ? __ldg(a.rho0detJ0 + z * N3 + qb) : ub[Dm::O_R + qb];
    double ga[9], gb[9];
#pragma unroll
    for (int i = 0; i < 9; ++i) { ga[i] = 0.0; gb[i] = 0.0; }
#pragma unroll
    for (int a0 = 0; a0 < (NOCV ? 1 : P); ++a0) {
      const double ba = tB[q0a * P + a0], gga = tG[q0a * P + a0];
      const double bb = tB[(q0a + NH) * P + a0], ggb = tG[(q0a + NH) * P + a0];
#pragma unroll
      for (int f = 0; f < 3; ++f)
#pragma unroll
        for (int m = 0; m < 3; ++m) {
          const double u = ub[(f * 3 + m) * UM + q2 * UQ + q1 * UQ1 + a0];
          ga[f * 3 + m] = fma(m == 0 ? gga : ba, u, ga[f * 3 + m]);
          gb[f * 3 + m] = fma(m == 0 ? ggb : bb, u, gb[f * 3 + m]);
        }
    }
    double ea = 0.0, eb = 0.0;
#pragma unroll
    for (int j0 = 0; j0 < T; ++j0) {
      const double ue = ub[Dm::O_UE + q2 * UQE + q1 * T + j0];
      ea = fma(tPhi[q0a * T + j0], ue, ea);
      eb = fma(tPhi[(q0a + NH) * T + j0], ue, eb);
    }
    if (PFENCE & 1) pfence(0);
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
    if (EARLYS && VMODE == 3 && a.ph.use_visc && a.ph.use_vort) {
      point_eval3<2, 1, EIG>(Ja, Gva, ea, Ra, sW[q0a] * w12, gamma, js, a.ph, oa, best);
#pragma unroll
      for (int cd = 0; cd < 9; ++cd) jb[cd * N3 + sa] = oa.S[cd / 3][cd % 3];
      jb[Dm::O_PQ + sa] = oa.P;
      point_eval3<2, 1, EIG>(Jb, Gvb, eb, Rb, sW[q0a + NH] * w12, gamma, js, a.ph, ob, best);
#pragma unroll
      for (int cd = 0; cd < 9; ++cd) jb[cd * N3 + sbi] = ob.S[cd / 3][cd % 3];
      jb[Dm::O_PQ + sbi] = ob.P;
      if (__any_sync(0xffffffffu, oa.cand || ob.cand)) {
        point_dt_exact_m(oa.m, a.ph, oa);
        point_dt_exact_m(ob.m, a.ph, ob);
      }
    } else if (VMODE == 3 && a.ph.use_visc && a.ph.use_vort) {   // both points one straight-line block, one vote
      const double la = KWB ? jb[Dm::O_PQ + sa] : 0.0, lb = KWB ? jb[Dm::O_PQ + sbi] : 0.0;
      point_eval3<2, 1, EIG, KWB ? 1 : 0>(Ja, Gva, ea, Ra, sW[q0a] * w12, gamma, js, a.ph, oa, best, 0xffffffffu, la);
      point_eval3<2, 1, EIG, KWB ? 1 : 0>(Jb, Gvb, eb, Rb, sW[q0a + NH] * w12, gamma, js, a.ph, ob, best, 0xffffffffu, lb);
      const bool anyc = __any_sync(0xffffffffu, oa.cand || ob.cand);
      if (DIAG == 4) { nvote4 += 1; nexact4 += anyc ? 1 : 0; }   // DIAG 4 (counting only): how often the exact dt runs
      if (DTX != 1 && (DTX == 2 || anyc)) {   // J is still in the JS buffer (S is written below)
        double Jr[3][3];
#pragma unroll
        for (int cd = 0; cd < 9; ++cd) Jr[cd / 3][cd % 3] = jb[cd * N3 + sa];
        point_dt_exact(Jr, a.ph, oa);
#pragma unroll
        for (int cd = 0; cd < 9; ++cd) Jr[cd / 3][cd % 3] = jb[cd * N3 + sbi];
        point_dt_exact(Jr, a.ph, ob);
      }
    } else if (VMODE == 1 || (VMODE >= 2 && a.ph.use_visc && a.ph.use_vort)) {   // production switches
      point_eval3<true, 1>(Ja, Gva, ea, Ra, sW[q0a] * w12, gamma, js, a.ph, oa, best);
      point_eval3<true, 1>(Jb, Gvb, eb, Rb, sW[q0a + NH] * w12, gamma, js, a.ph, ob, best);
    } else {
      point_eval3<true>(Ja, Gva, ea, Ra, sW[q0a] * w12, gamma, js, a.ph, oa, best);
      point_eval3<true>(Jb, Gvb, eb, Rb, sW[q0a + NH] * w12, gamma, js, a.ph, ob, best);
    }
    {
      double mi = fmax(oa.inv, ob.inv);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) mi = fmax(mi, __shfl_xor_sync(0xffffffffu, mi, o));
      if ((threadIdx.x & 31) == 0 && mi > best)
        atomicMax(reinterpret_cast<unsigned long long *>(sRed + 8), (unsigned long long)__double_as_longlong(mi));
    }
    if (DIAG == 3 && !PCT) {   // keep S live without overwriting J (a store that never happens)
      double acc = oa.P + ob.P;
#pragma unroll
      for (int cd = 0; cd < 9; ++cd) acc += oa.S[cd / 3][cd % 3] + ob.S[cd / 3][cd % 3];
      if (acc == 1.2345e300) jb[Dm::O_PQ + sa] = acc;
    } else if (PCT) {
      if (PFENCE & 2) pfence(1);
      static_assert(N == 8 && P <= 8 && T <= 8 && NPW == 256, "PCT: one m8n8k4 tile per (warp, field), k-steps = q0 halves");
      const int ln = tid & 31, lr = ln >> 2, lc = ln & 3;   // lr = q1, lc = q0a (pr = tid)
      // A fragments: table^T[a = lr][q0 = 4 s + lc] (rows a >= P / T are zero)
      const double fb0 = lr < P ? tB[lc * P + lr] : 0.0, fb1 = lr < P ? tB[(lc + 4) * P + lr] : 0.0;
      const double fg0 = lr < P ? tG[lc * P + lr] : 0.0, fg1 = lr < P ? tG[(lc + 4) * P + lr] : 0.0;
      const double fp0 = lr < T ? tPhi[lc * T + lr] : 0.0, fp1 = lr < T ? tPhi[(lc + 4) * T + lr] : 0.0;
      __syncwarp();   // every lane's J (re)reads of this warp's rows precede the Y stores over them
      double *yw = (DIAG == 3 ? sWk : jb) + q2 * N2 + lr * N + 2 * lc;   // DIAG 3: J must survive (timing only)
#pragma unroll
      for (int cd = 0; cd < NPC; ++cd) {
        double d0 = 0.0, d1 = 0.0;
        const double sa_ = cd < 9 ? oa.S[cd / 3][cd % 3] : oa.P, sb_ = cd < 9 ? ob.S[cd / 3][cd % 3] : ob.P;
        dmma(d0, d1, cd == 9 ? fp0 : (cd % 3 == 0 ? fg0 : fb0), sa_);
        dmma(d0, d1, cd == 9 ? fp1 : (cd % 3 == 0 ? fg1 : fb1), sb_);
        if (lr < (cd == 9 ? T : P)) sts_f64x2(yw + cd * N3, d0, d1);
      }
#pragma unroll
      for (int cd = NPC; cd < 9; ++cd) {   // the contraction warps' fields: S in place over J
        jb[cd * N3 + sa] = oa.S[cd / 3][cd % 3];
        jb[cd * N3 + sbi] = ob.S[cd / 3][cd % 3];
      }
      if (NPC < 10) {
        jb[Dm::O_PQ + sa] = oa.P;
        jb[Dm::O_PQ + sbi] = ob.P;
      }
    } else if (!(EARLYS && VMODE == 3 && a.ph.use_visc && a.ph.use_vort)) {
#pragma unroll
      for (int cd = 0; cd < 9; ++cd) {     // in place over J: only this thread touches slots sa, sbi
        jb[cd * N3 + sa] = oa.S[cd / 3][cd % 3];
        jb[cd * N3 + sbi] = ob.S[cd / 3][cd % 3];
      }
      jb[Dm::O_PQ + sa] = oa.P;
      jb[Dm::O_PQ + sbi] = ob.P;
    }
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
    if (BULK && tid == NPW) {
      mbar_init(sMB, 1);
      mbar_init(sMB + 1, 1);
      asm volatile("fence.mbarrier_init.release.cluster;\nfence.proxy.async.shared::cta;\n" ::: "memory");
    }
    if (FF) {   // node gather of zone zi into XEb[zi & 1]; rho0|J0| of zone zr into UV[zr & 1]
      auto ff_nodes = [&](int64_t zi) {
        if (zi >= nz) return;
        const int64_t z = zone_of(zi);
        double *xe = sXEb[zi & 1];
        if (ktid < P3) {
          const int64_t node = sID[(zi & 1) * P3 + ktid];
#pragma unroll
          for (int c = 0; c < 3; ++c) {
            cp_async8(xe + Dm::XE_X + c * P3 + ktid, a.x + c * nn + node, true);
            cp_async8(xe + Dm::XE_X + (3 + c) * P3 + ktid, a.v + c * nn + node, true);
          }
        }
        for (int r = ktid; r < T3 + 10; r += NKW) {
          const double *src = r < T3 ? a.e + z * T3 + r : r < T3 + 9 ? a.J0inv + z * 9 + (r - T3) : a.zone_gamma + z;
          cp_async8(xe + Dm::XE_E + r, src, true);
        }
      };
      auto ff_rho = [&](int64_t zr) {
        if (zr >= nz) return;
        double *R = sUV + (zr & 1) * Dm::UVBUF + Dm::O_R;
        const int64_t z = zone_of(zr);
        for (int r = ktid; r < N3; r += NKW) cp_async8(R + r, a.rho0detJ0 + z * N3 + r, true);
      };
      kw_load_id(0);
      kw_load_id(1);
      cp_async_commit();
      cp_async_wait<0>();
      kw_bar<NKW>();
      ff_nodes(0);
      ff_rho(0);
      ff_nodes(1);
      kw_load_id(2);
      cp_async_commit();
      cp_async_wait<0>();
      kw_bar<NKW>();
      if (nz > 0) kw_forward(sUV, sJS, sJ, a.zero, sXEb[0]);
      cta_bar_div<Cfg::NTH>();
      long long t_work = 0;
      int itc = 2;
      for (int64_t i = 0; i <= nz; ++i, ++itc) {
        const long long t0 = CLK ? clock64() : 0;
        ff_nodes(i + 2);
        ff_rho(i + 1);
        kw_load_id(i + 3);
        cp_async_commit();
        kstamp(3);
        const int zc = a.zero * itc;
        const bool fw = i + 1 < nz, back = i >= 1;
        double *ub1 = sUV + ((i + 1) & 1) * Dm::UVBUF, *jb1 = sJS + ((i + 1) & 1) * Dm::JSBUF, *js1 = sJ + ((i + 1) & 1) * 10;
        if (fw) kw_forward(ub1, jb1, js1, zc + a.zero, sXEb[(i + 1) & 1], 1);   // A, B (ends with a KW barrier)
        if (back) kw_back(sJS + ((i - 1) & 1) * Dm::JSBUF, zone_of(i - 1), zc, [] {}, 1);   // B^T (ends with a barrier)
        if (fw) kw_forward(ub1, jb1, js1, zc + a.zero, sXEb[(i + 1) & 1], 2);   // C_x: J(i+1) over Y(i-1), read by B^T
        if (back) kw_back(sJS + ((i - 1) & 1) * Dm::JSBUF, zone_of(i - 1), zc, [] {}, 2);   // A^T (+ KW barrier)
        cp_async_wait<0>();   // zone i+2's nodes, zone i+1's rho0|J0| (read by the point warps next period)
        if (CLK) t_work += clock64() - t0;
        cta_bar_div<Cfg::NTH>();
        kstamp(11);
      }
      if (a.prof != nullptr && tid == NPW) {
        a.prof[blockIdx.x * 16 + 1] = t_work;
        for (int sl = 3; sl < 12; ++sl) a.prof[blockIdx.x * 16 + sl] = sKP[sl];
      }
      return;
    }
    if (PWG) {   // the point warps issue the gathers
      if (nz > 0) mbar_wait(sMB, 0u);
    } else {
      kw_load_id(0);
      cp_async_commit();
      cp_async_wait<0>();
      kw_bar<NKW>();                 // ids of zone 0 (and the mbarrier init)
      kw_issue(0);
      kw_load_id(1);
      cp_async_commit();
      cp_async_wait<0>();
      kw_wait_bulk(0);
    }
    kw_bar<NKW>();
    if (nz > 0 && DIAG != 1) kw_forward(sUV, sJS, sJ, a.zero, sXEb[0]);
    cta_bar_div<Cfg::NTH>();
    long long t_work = 0;
    int itc = 2;
    for (int64_t i = 0; i <= nz; ++i, ++itc) {
      const long long t0 = CLK ? clock64() : 0;
      auto issue = [&] {
        kw_issue(i + 1);
        kw_load_id(i + 2);
        cp_async_commit();
      };
      // DIAG 3 (timing only): the point warps alone on valid data -- zones 0 and 1 are formed once, nothing else
      const bool back = i >= 1 && DIAG != 1 && DIAG != 3;
      if (KSLEEP > 0 && back) __nanosleep(KSLEEP);   // timing experiment: let the point warps' stage C_v start alone
      if (!PWG && !(LATE && back)) issue();
      kstamp(3);
      const int zc = a.zero * itc;   // 0, but loop-variant and uniform
      if (back) kw_back(sJS + ((i - 1) & 1) * Dm::JSBUF, zone_of(i - 1), zc, [&] { if (LATE) issue(); });
      if (PWG) {
        if (i + 1 < nz) mbar_wait(sMB + ((i + 1) & 1), (unsigned)(((i + 1) >> 1) & 1));
      } else {
        cp_async_wait<0>();
        kw_wait_bulk(i + 1);
      }
      kw_bar<NKW>();
      kstamp(7);
      if (i + 1 < nz && DIAG != 1 && (DIAG != 3 || i + 1 < 2))
        kw_forward(sUV + ((i + 1) & 1) * Dm::UVBUF, sJS + ((i + 1) & 1) * Dm::JSBUF, sJ + ((i + 1) & 1) * 10, zc + a.zero,
                   PWG ? sXEb[(i + 1) & 1] : sXE);
      if (CLK) t_work += clock64() - t0;
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
  // PWG: the gather of zone zi (node ids one zone earlier), issued by the point warps; every point thread
  // arrives once per zone on mbarrier zi & 1 when its copies have landed.  A thread copies rho0|J0| of
  // exactly its own two points, so it never overwrites an entry another thread has still to read.
  auto pw_load_id = [&](int64_t zi) {
    if (zi < nz && tid < P3) cp_async4(sID + (zi & 1) * P3 + tid, a.zone_nodes + zone_of(zi) * P3 + tid);
  };
  auto pw_issue = [&](int64_t zi) {
    if (zi >= nz) return;
    const int64_t z = zone_of(zi);
    double *xe = sXEb[zi & 1];
    if (tid < P3) {
      const int64_t node = sID[(zi & 1) * P3 + tid];
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        cp_async8(xe + Dm::XE_X + c * P3 + tid, a.x + c * nn + node, true);
        cp_async8(xe + Dm::XE_X + (3 + c) * P3 + tid, a.v + c * nn + node, true);
      }
    } else if (tid < P3 + T3 + 10) {
      const int r = tid - P3;
      const double *src = r < T3 ? a.e + z * T3 + r : r < T3 + 9 ? a.J0inv + z * 9 + (r - T3) : a.zone_gamma + z;
      cp_async8(xe + Dm::XE_E + r, src, true);
    }
    if (tid < TPZ) {
      const int qa = (q2 * N + q1) * N + q0a;
      double *R = sUV + (zi & 1) * Dm::UVBUF + Dm::O_R;
      cp_async8(R + qa, a.rho0detJ0 + z * N3 + qa, true);
      cp_async8(R + qa + NH, a.rho0detJ0 + z * N3 + qa + NH, true);
    }
    cp_async_mbar_arrive(sMB + (zi & 1));
  };
  if (PWG) {
    pw_load_id(0);
    pw_load_id(1);
    cp_async_commit();
    cp_async_wait<0>();   // each thread reads back only the ids it loaded
    pw_issue(0);
    pw_issue(1);
    pw_load_id(2);
    cp_async_commit();
  }
  cta_bar_div<Cfg::NTH>();
  long long t_work = 0, t_all = CLK ? clock64() : 0;
  for (int64_t i = 0; i <= nz; ++i) {
    const long long t0 = CLK ? clock64() : 0;
    if (RHOPW && i + 1 < nz && tid < TPZ) {   // zone i+1's rho0|J0| lines into L2
      const double *rz = a.rho0detJ0 + zone_of(i + 1) * N3;
      if ((tid & 7) == 0) asm volatile("prefetch.global.L2 [%0];" ::"l"(rz + 2 * tid));   // 32 lines of 16 doubles
    }
    if (i < nz && tid < TPZ && DIAG != 2)
      pw_point(sUV + (i & 1) * Dm::UVBUF, sJ + (i & 1) * 10, sJS + (i & 1) * Dm::JSBUF, zone_of(i));
    if (PWG) {   // zone i's points are done: issue zone i+2 (its XE and R slots were last read for zone i)
      cp_async_wait<0>();
      pw_issue(i + 2);
      pw_load_id(i + 3);
      cp_async_commit();
    }
    if (CLK) t_work += clock64() - t0;
    cta_bar_div<Cfg::NTH>();
  }
  if (PWG) cp_async_wait<0>();
  if (a.prof != nullptr && tid == 0) {
    a.prof[blockIdx.x * 16 + 0] = t_work;
    a.prof[blockIdx.x * 16 + 2] = clock64() - t_all;
  }
  if (DIAG == 4 && a.prof != nullptr && (tid & 31) == 0 && tid < NPW) {
    atomicAdd(reinterpret_cast<unsigned long long *>(a.prof + blockIdx.x * 16 + 12), (unsigned long long)nvote4);
    atomicAdd(reinterpret_cast<unsigned long long *>(a.prof + blockIdx.x * 16 + 13), (unsigned long long)nexact4);
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
