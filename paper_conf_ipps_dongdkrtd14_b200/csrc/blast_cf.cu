// libblastcf.so — host library and C ABI (include/blast_cf.h) of the B200 corner-force path.
//
// create(): validates the mesh, builds the 1-D tables (tables.h), the per-zone J0^{-1} of the affine
// initial zones and h0, the inverse node -> (zone, local) CSR in ascending zone id, uploads everything
// and sizes the launch.  eval(): KB1 (kb1_corner_force.cuh) then KB2 (kb2_gather.cuh) on the handle's
// stream, plus the shared-DOF exchange when nranks > 1 (exchange.cuh).  No allocation in eval.
#include <cuda_runtime.h>

#include <unistd.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "../../include/blast_cf.h"
#include <nvtx3/nvToolsExt.h>   // header-only NVTX v3: ranges cost nothing unless a tool (nsys, ncu) is attached
#include "kb1_corner_force.cuh"
#include "kb1_v2.cuh"
#include "kb1_v3.cuh"
#include "kb1_v4.cuh"
#include "kb1_v5.cuh"
#include "kb1_v6.cuh"
#include "kb1_v10.cuh"
#include "kb1_v8.cuh"
#include "kb1_v11.cuh"
#include "kb1_p2d.cuh"
#include "kb2_gather.cuh"
#include "tables.h"
#include "exchange.cuh"
#include "internal.h"

namespace {

thread_local std::string g_last_error;

// NVTX range for the host-side phases (tracing); the kernels themselves are visible to the tools
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

int fail(int code, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return code;
}

#define CUDA_TRY(expr)                                                                       \
  do {                                                                                       \
    cudaError_t e_ = (expr);                                                                 \
    if (e_ != cudaSuccess)                                                                   \
      return fail(e_ == cudaErrorMemoryAllocation ? BLAST_CF_ENOMEM : BLAST_CF_ECUDA,        \
                  "%s: %s (%s:%d)", #expr, cudaGetErrorString(e_), __FILE__, __LINE__);      \
  } while (0)

template <typename T>
int upload(T **dst, const T *src, size_t count) {
  CUDA_TRY(cudaMalloc((void **)dst, std::max<size_t>(count, 1) * sizeof(T)));
  if (count) CUDA_TRY(cudaMemcpy(*dst, src, count * sizeof(T), cudaMemcpyHostToDevice));
  return BLAST_CF_OK;
}

// ------------------------------------------------------------------------------------------------
// kernel instantiation table: (dim, k) -> zones per CTA, threads, shared memory, launcher
// ------------------------------------------------------------------------------------------------
typedef void (*kb1_launch_fn)(const KB1Args &, int grid, cudaStream_t);

struct KB1Variant {
  int zpc, nth, smem;
  kb1_launch_fn launch;
  const void *func;
  bool persistent;   // grid = resident CTAs; CTA c runs zone batches c, c + grid, ...
  const char *name = nullptr;
  bool point_j0 = false;   // reads KB1Args::J0inv_q (per-point J0^{-1} of non-affine initial meshes)
};

template <int K, int ZPC, int MINB>
void launch3(const KB1Args &a, int grid, cudaStream_t s) {
  using C = KB1Cfg3<K, ZPC>;
  kb1_corner_force_3d<K, ZPC, MINB><<<grid, C::NTH, C::SMEM_BYTES, s>>>(a);
}
template <int K, int ZPC, int MINB>
void launch2(const KB1Args &a, int grid, cudaStream_t s) {
  using C = KB1Cfg2<K, ZPC>;
  kb1_corner_force_2d<K, ZPC, MINB><<<grid, C::NTH, C::SMEM_BYTES, s>>>(a);
}
template <int K, int ZPC, int MINB, int PPT, int EX>
void launch3v2(const KB1Args &a, int grid, cudaStream_t s) {
  using C = KB1V2Cfg<K, ZPC, PPT>;
  kb1_v2_3d<K, ZPC, MINB, PPT, EX><<<grid, C::NTH, C::SMEM_BYTES, s>>>(a);
}
template <int K, int ZPC, int MINB, int PPT = 2, int EX = 0>
KB1Variant variant3v2() {
  using C = KB1V2Cfg<K, ZPC, PPT>;
  return KB1Variant{ZPC, C::NTH, C::SMEM_BYTES, &launch3v2<K, ZPC, MINB, PPT, EX>,
                    (const void *)&kb1_v2_3d<K, ZPC, MINB, PPT, EX>, true, nullptr};
}
template <int K, int ZPC, int MINB>
void launch3v3(const KB1Args &a, int grid, cudaStream_t s) {
  using C = KB1V3Cfg<K, ZPC>;
  kb1_v3_3d<K, ZPC, MINB><<<grid, C::NTH, C::SMEM_BYTES, s>>>(a);
}
template <int K, int ZPC, int MINB>
KB1Variant variant3v3() {
  using C = KB1V3Cfg<K, ZPC>;
  return KB1Variant{ZPC, C::NTH, C::SMEM_BYTES, &launch3v3<K, ZPC, MINB>, (const void *)&kb1_v3_3d<K, ZPC, MINB>,
                    false, nullptr};
}
template <int K, int DIAG, int MODE>
void launch3v5(const KB1Args &a, int grid, cudaStream_t s) {
  using C = KB1V5Cfg<K, MODE>;
  kb1_v5_3d<K, DIAG, MODE><<<grid, C::NTH, C::SMEM_BYTES, s>>>(a);
}
template <int K, int DIAG = 0, int MODE = 0>
KB1Variant variant3v5() {
  using C = KB1V5Cfg<K, MODE>;
  return KB1Variant{1, C::NTH, C::SMEM_BYTES, &launch3v5<K, DIAG, MODE>, (const void *)&kb1_v5_3d<K, DIAG, MODE>,
                    true, nullptr};
}
template <int K, int DIAG, int MODE, int OPT, int VMODE>
void launch3v10(const KB1Args &a, int grid, cudaStream_t s) {
  using C = KB1V5Cfg<K, MODE>;
  kb1_v10_3d<K, DIAG, MODE, OPT, VMODE><<<grid, C::NTH, v10_smem_bytes<K, OPT>(), s>>>(a);
}
template <int K, int DIAG = 0, int MODE = 0, int OPT = 0, int VMODE = 0>
KB1Variant variant3v10() {
  using C = KB1V5Cfg<K, MODE>;
  return KB1Variant{1, C::NTH, v10_smem_bytes<K, OPT>(), &launch3v10<K, DIAG, MODE, OPT, VMODE>,
                    (const void *)&kb1_v10_3d<K, DIAG, MODE, OPT, VMODE>, true, nullptr};
}
template <int K, int MINB>
void launch3v8(const KB1Args &a, int grid, cudaStream_t s) {
  using C = KB1V8Cfg<K>;
  kb1_v8_3d<K, MINB><<<grid, C::NTH, C::SMEM_BYTES, s>>>(a);
}
template <int K, int MINB>
KB1Variant variant3v8() {
  using C = KB1V8Cfg<K>;
  return KB1Variant{1, C::NTH, C::SMEM_BYTES, &launch3v8<K, MINB>, (const void *)&kb1_v8_3d<K, MINB>, false, nullptr};
}
template <int K, int MINB, int MB>
void launch3v11(const KB1Args &a, int grid, cudaStream_t s) {
  using C = KB1V11Cfg<K>;
  kb1_v11_3d<K, MINB, MB><<<grid, C::NTH, C::SMEM_BYTES, s>>>(a);
}
template <int K, int MINB, int MB = 0>
KB1Variant variant3v11() {
  using C = KB1V11Cfg<K>;
  return KB1Variant{1, C::NTH, C::SMEM_BYTES, &launch3v11<K, MINB, MB>, (const void *)&kb1_v11_3d<K, MINB, MB>, true,
                    nullptr};
}
template <int K, int ZPC, int MINB>
KB1Variant variant3() {
  using C = KB1Cfg3<K, ZPC>;
  return KB1Variant{ZPC, C::NTH, C::SMEM_BYTES, &launch3<K, ZPC, MINB>,
                    (const void *)&kb1_corner_force_3d<K, ZPC, MINB>, false, nullptr, true};
}
template <int K, int ZPC, int MINB>
void launchP2d(const KB1Args &a, int grid, cudaStream_t s) {
  using C = KB1CfgP2d<K, ZPC>;
  kb1_p2d<K, ZPC, MINB><<<grid, C::NTH, C::SMEM_BYTES, s>>>(a);
}
template <int K, int ZPC, int MINB>
KB1Variant variantP2d() {
  using C = KB1CfgP2d<K, ZPC>;
  return KB1Variant{ZPC, C::NTH, C::SMEM_BYTES, &launchP2d<K, ZPC, MINB>, (const void *)&kb1_p2d<K, ZPC, MINB>, true,
                    nullptr};
}
template <int K, int ZPC, int MINB>
KB1Variant variant2() {
  using C = KB1Cfg2<K, ZPC>;
  return KB1Variant{ZPC, C::NTH, C::SMEM_BYTES, &launch2<K, ZPC, MINB>,
                    (const void *)&kb1_corner_force_2d<K, ZPC, MINB>, false, nullptr, true};
}

// Candidate KB1 variants per (dim, k), default first (f3 of SURVEY §8: the create-time default is the
// measured winner of round 1; blast_cf_autotune re-times all candidates on the caller's data).
std::vector<KB1Variant> kb1_candidates(int dim, int k) {
  std::vector<KB1Variant> v;
  auto add = [&](KB1Variant x, const char *name) { x.name = name; v.push_back(x); };
  if (dim == 3) {
    switch (k) {
      case 1: add(variant3v2<1, 32, 2, 1>(), "v2.p1.z32"); add(variant3v2<1, 64, 2>(), "v2.z64"); add(variant3<1, 32, 2>(), "v1.z32"); break;
      case 2: add(variant3v2<2, 1, 12, 2, 6>(), "v2.z1m12e"); add(variant3v2<2, 1, 12>(), "v2.z1m12"); add(variant3v2<2, 2, 6>(), "v2.z2m6"); add(variant3v2<2, 2, 4, 1>(), "v2.p1.z2"); add(variant3<2, 16, 2>(), "v1.z16"); break;
      case 3: add(variant3v2<3, 2, 2>(), "v2.z2"); add(variant3v2<3, 1, 2, 1>(), "v2.p1.z1"); add(variant3v3<3, 2, 2>(), "v3.z2"); add(variant3<3, 8, 2>(), "v1.z8"); break;
      case 4:
        // (round 2: the superseded generations v10 (runtime switches), v10.wu, v6, v5, v4.m0/m1, v3.z1 that never
        //  won the autotuner are no longer instantiated; DESIGN.md §10 keeps their measurements)
        add(variant3v10<4, 0, 0, (1 << 25), 3 | 8>(), "v10.wpx");
        add(variant3v10<4, 0, 0, 0, 3>(), "v10.w");
        add(variant3v10<4, 0, 0, 0, 2>(), "v10.v"); add(variant3v5<4, 0, 1>(), "v5.r1");
        add(variant3v2<4, 1, 2>(), "v2.z1"); add(variant3<4, 4, 2>(), "v1.z4");
        break;
      case 5: add(variant3<5, 2, 2>(), "v1.z2"); break;
      case 6: add(variant3<6, 1, 2>(), "v1.z1m2"); add(variant3<6, 2, 1>(), "v1.z2"); break;
      case 7: add(variant3v8<7, 1>(), "v8"); add(variant3v11<7, 1>(), "v11"); add(variant3<7, 1, 2>(), "v1.z1"); break;
      case 8: add(variant3v11<8, 2, 83 | 128 | 256>(), "v11.mbtsiet"); add(variant3v11<8, 2, 83 | 128>(), "v11.mbtsie"); add(variant3v11<8, 2, 83>(), "v11.mbtsi"); add(variant3v11<8, 2, 19>(), "v11.mbts"); add(variant3v11<8, 2, 3>(), "v11.mbt"); add(variant3v11<8, 2, 1>(), "v11.mb"); add(variant3v8<8, 2>(), "v8"); add(variant3v11<8, 2>(), "v11"); add(variant3v8<8, 1>(), "v8.m1"); add(variant3<8, 1, 2>(), "v1.z1m2"); add(variant3<8, 1, 1>(), "v1.z1"); break;
    }
  } else {
    switch (k) {
      case 1: add(variant2<1, 64, 2>(), "v1-2d.z64"); break;
      case 2: add(variant2<2, 16, 2>(), "v1-2d.z16"); break;
      case 3: add(variant2<3, 8, 2>(), "v1-2d.z8"); break;
      case 4: add(variantP2d<4, 2, 6>(), "p2d.z2m6"); add(variantP2d<4, 4, 3>(), "p2d.z4m3"); add(variant2<4, 4, 3>(), "v1-2d.z4m3"); add(variant2<4, 4, 2>(), "v1-2d.z4"); break;
      case 5: add(variant2<5, 2, 2>(), "v1-2d.z2"); break;
      case 6: add(variant2<6, 2, 2>(), "v1-2d.z2"); break;
      case 7: add(variant2<7, 1, 2>(), "v1-2d.z1"); break;
      case 8: add(variant2<8, 1, 2>(), "v1-2d.z1"); break;
    }
  }
  return v;
}

// the candidates a handle may use: all of them, or (non-affine initial mesh) those that read J0inv_q
std::vector<KB1Variant> kb1_usable(int dim, int k, bool need_point_j0) {
  std::vector<KB1Variant> c = kb1_candidates(dim, k);
  if (need_point_j0) c.erase(std::remove_if(c.begin(), c.end(), [](const KB1Variant &x) { return !x.point_j0; }), c.end());
  return c;
}

KB1Variant select_variant(int dim, int k, bool need_point_j0) {
  const std::vector<KB1Variant> c = kb1_usable(dim, k, need_point_j0);
  if (c.empty()) return KB1Variant{0, 0, 0, nullptr, nullptr, false, nullptr};
  const char *force = getenv("BLAST_CF_KB1");   // experiments: pick a candidate by name
  if (force) {
    for (const KB1Variant &x : c)
      if (strcmp(x.name, force) == 0) return x;
#ifdef BLAST_CF_DIAGNOSTICS
    if (need_point_j0) return c[0];
    // timing diagnostics (wrong results by design; never candidates of the autotuner): compiled only into a
    // -DBLAST_CF_DIAGNOSTICS build, never into the production library
    if (dim == 3 && k == 2) {
      KB1Variant d;
      if (strcmp(force, "v2.p1.z2e") == 0) { d = variant3v2<2, 2, 4, 1, 6>(); d.name = "v2.p1.z2e"; return d; }
      if (strcmp(force, "v2.p1.z2m5e") == 0) { d = variant3v2<2, 2, 5, 1, 6>(); d.name = "v2.p1.z2m5e"; return d; }
      if (strcmp(force, "v2.p1.z1m8e") == 0) { d = variant3v2<2, 1, 8, 1, 6>(); d.name = "v2.p1.z1m8e"; return d; }
      if (strcmp(force, "v2.p1.z1m10e") == 0) { d = variant3v2<2, 1, 10, 1, 6>(); d.name = "v2.p1.z1m10e"; return d; }
      if (strcmp(force, "v2.z1m13e") == 0) { d = variant3v2<2, 1, 13, 2, 6>(); d.name = "v2.z1m13e"; return d; }
      if (strcmp(force, "v2.z1m11e") == 0) { d = variant3v2<2, 1, 11, 2, 6>(); d.name = "v2.z1m11e"; return d; }
    }
    if (dim == 3 && k == 8) {
      KB1Variant d;
      if (strcmp(force, "v11.mbtcie") == 0) { d = variant3v11<8, 2, 83 | 128 | 4>(); d.name = "v11.mbtcie"; return d; }
      if (strcmp(force, "v11.mbtce") == 0) { d = variant3v11<8, 2, 19 | 128 | 4>(); d.name = "v11.mbtce"; return d; }
      if (strcmp(force, "v11.mbtse") == 0) { d = variant3v11<8, 2, 19 | 128>(); d.name = "v11.mbtse"; return d; }
    }
    if (dim == 3 && k == 4) {
      KB1Variant d;
      if (strcmp(force, "v5.d1") == 0) { d = variant3v5<4, 1>(); d.name = "v5.d1"; return d; }
      if (strcmp(force, "v5.d2") == 0) { d = variant3v5<4, 2>(); d.name = "v5.d2"; return d; }
      if (strcmp(force, "v10.q") == 0) { d = variant3v10<4, 0, 0, 4>(); d.name = "v10.q"; return d; }
      if (strcmp(force, "v10.b") == 0) { d = variant3v10<4, 0, 0, 1>(); d.name = "v10.b"; return d; }
      if (strcmp(force, "v10.l") == 0) { d = variant3v10<4, 0, 0, 2>(); d.name = "v10.l"; return d; }
      if (strcmp(force, "v10.w16") == 0) { d = variant3v10<4, 0, 0, 16, 3>(); d.name = "v10.w16"; return d; }
      if (strcmp(force, "v10.x") == 0) { d = variant3v10<4, 0, 0, 8, 3>(); d.name = "v10.x"; return d; }
      if (strcmp(force, "v10.xd1") == 0) { d = variant3v10<4, 1, 0, 8, 3>(); d.name = "v10.xd1"; return d; }
      if (strcmp(force, "v10.xd2") == 0) { d = variant3v10<4, 2, 0, 8, 3>(); d.name = "v10.xd2"; return d; }
      if (strcmp(force, "v10.wq") == 0) { d = variant3v10<4, 0, 0, 4, 3>(); d.name = "v10.wq"; return d; }
      if (strcmp(force, "v10.wl") == 0) { d = variant3v10<4, 0, 0, 2, 3>(); d.name = "v10.wl"; return d; }
      if (strcmp(force, "v10.we") == 0) { d = variant3v10<4, 0, 0, 512, 3>(); d.name = "v10.we"; return d; }
      if (strcmp(force, "v10.wr1") == 0) { d = variant3v10<4, 0, 1, 0, 3>(); d.name = "v10.wr1"; return d; }
      if (strcmp(force, "v10.wn") == 0) { d = variant3v10<4, 0, 0, 2048, 3>(); d.name = "v10.wn"; return d; }
      if (strcmp(force, "v10.wpad") == 0) { d = variant3v10<4, 0, 0, 1024, 3>(); d.name = "v10.wpad"; return d; }
      if (strcmp(force, "v10.ws") == 0) { d = variant3v10<4, 0, 0, 64, 3>(); d.name = "v10.ws"; return d; }
      if (strcmp(force, "v10.wnoxv") == 0) { d = variant3v10<4, 0, 0, 32, 3>(); d.name = "v10.wnoxv"; return d; }
      if (strcmp(force, "v10.wr4") == 0) { d = variant3v10<4, 0, 4, 0, 3>(); d.name = "v10.wr4"; return d; }
      if (strcmp(force, "v10.wr3") == 0) { d = variant3v10<4, 0, 3, 0, 3>(); d.name = "v10.wr3"; return d; }
      if (strcmp(force, "v10.wd1") == 0) { d = variant3v10<4, 1, 0, 0, 3>(); d.name = "v10.wd1"; return d; }
      if (strcmp(force, "v10.vd1") == 0) { d = variant3v10<4, 1, 0, 0, 2>(); d.name = "v10.vd1"; return d; }
      if (strcmp(force, "v10.d1") == 0) { d = variant3v10<4, 1>(); d.name = "v10.d1"; return d; }
      if (strcmp(force, "v10.wdt0") == 0) { d = variant3v10<4, 0, 0, 131072, 3>(); d.name = "v10.wdt0"; return d; }
      if (strcmp(force, "v10.wdt1") == 0) { d = variant3v10<4, 0, 0, 262144, 3>(); d.name = "v10.wdt1"; return d; }
      if (strcmp(force, "v10.wnc") == 0) { d = variant3v10<4, 0, 0, 524288, 3>(); d.name = "v10.wnc"; return d; }
      if (strcmp(force, "v10.wd2") == 0) { d = variant3v10<4, 2, 0, 0, 3>(); d.name = "v10.wd2"; return d; }
      if (strcmp(force, "v10.wd3") == 0) { d = variant3v10<4, 3, 0, 0, 3>(); d.name = "v10.wd3"; return d; }
      if (strcmp(force, "v10.wd3nc") == 0) { d = variant3v10<4, 3, 0, 524288, 3>(); d.name = "v10.wd3nc"; return d; }
      if (strcmp(force, "v10.wd3ne") == 0) { d = variant3v10<4, 3, 0, 2097152, 3>(); d.name = "v10.wd3ne"; return d; }
      if (strcmp(force, "v10.wd3ncv") == 0) { d = variant3v10<4, 3, 0, 1048576, 3>(); d.name = "v10.wd3ncv"; return d; }
      if (strcmp(force, "v10.wd3x") == 0) { d = variant3v10<4, 3, 0, 1048576 | 2097152, 3>(); d.name = "v10.wd3x"; return d; }
      if (strcmp(force, "v10.wskct") == 0) { d = variant3v10<4, 0, 0, (1 << 21), 3>(); d.name = "v10.wskct"; return d; }
      if (strcmp(force, "v10.wskba") == 0) { d = variant3v10<4, 0, 0, (1 << 22), 3>(); d.name = "v10.wskba"; return d; }
      if (strcmp(force, "v10.wskab") == 0) { d = variant3v10<4, 0, 0, (1 << 23), 3>(); d.name = "v10.wskab"; return d; }
      if (strcmp(force, "v10.wskcx") == 0) { d = variant3v10<4, 0, 0, (1 << 24), 3>(); d.name = "v10.wskcx"; return d; }
      if (strcmp(force, "v10.wk1") == 0) { d = variant3v10<4, 0, 0, (1 << 27), 3>(); d.name = "v10.wk1"; return d; }
      if (strcmp(force, "v10.wpk1") == 0) { d = variant3v10<4, 0, 0, (1 << 27) | (1 << 25), 3>(); d.name = "v10.wpk1"; return d; }
      if (strcmp(force, "v10.wk2") == 0) { d = variant3v10<4, 0, 0, (2 << 27), 3>(); d.name = "v10.wk2"; return d; }
      if (strcmp(force, "v10.wpk2") == 0) { d = variant3v10<4, 0, 0, (2 << 27) | (1 << 25), 3>(); d.name = "v10.wpk2"; return d; }
      if (strcmp(force, "v10.wk3") == 0) { d = variant3v10<4, 0, 0, (3 << 27), 3>(); d.name = "v10.wk3"; return d; }
      if (strcmp(force, "v10.wpk3") == 0) { d = variant3v10<4, 0, 0, (3 << 27) | (1 << 25), 3>(); d.name = "v10.wpk3"; return d; }
      if (strcmp(force, "v10.wxr4") == 0) { d = variant3v10<4, 0, 4, 0, 3 | 8>(); d.name = "v10.wxr4"; return d; }
      if (strcmp(force, "v10.wxr3") == 0) { d = variant3v10<4, 0, 3, 0, 3 | 8>(); d.name = "v10.wxr3"; return d; }
      if (strcmp(force, "v10.wpxr4") == 0) { d = variant3v10<4, 0, 4, (1 << 25), 3 | 8>(); d.name = "v10.wpxr4"; return d; }
      if (strcmp(force, "v10.wpxk1") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | (1 << 27), 3 | 8>(); d.name = "v10.wpxk1"; return d; }
      if (strcmp(force, "v10.wpxk2") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | (2 << 27), 3 | 8>(); d.name = "v10.wpxk2"; return d; }
      if (strcmp(force, "v10.wpxb") == 0) { d = variant3v10<4, 0, 0, (1 << 25), 3 | 8 | 16>(); d.name = "v10.wpxb"; return d; }
      if (strcmp(force, "v10.wpxd3") == 0) { d = variant3v10<4, 3, 0, (1 << 25), 3 | 8>(); d.name = "v10.wpxd3"; return d; }
      if (strcmp(force, "v10.wpxd2") == 0) { d = variant3v10<4, 2, 0, (1 << 25), 3 | 8>(); d.name = "v10.wpxd2"; return d; }
      if (strcmp(force, "v10.wpxncv") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | 1048576, 3 | 8>(); d.name = "v10.wpxncv"; return d; }
      if (strcmp(force, "v10.wpxnc") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | 524288, 3>(); d.name = "v10.wpxnc"; return d; }
      if (strcmp(force, "v10.wpxskba") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | (1 << 22), 3 | 8>(); d.name = "v10.wpxskba"; return d; }
      if (strcmp(force, "v10.wpxd4") == 0) { d = variant3v10<4, 4, 0, (1 << 25), 3 | 8>(); d.name = "v10.wpxd4"; return d; }
      if (strcmp(force, "v10.wpxr3") == 0) { d = variant3v10<4, 0, 3, (1 << 25), 3 | 8>(); d.name = "v10.wpxr3"; return d; }
      if (strcmp(force, "v10.wpxr1") == 0) { d = variant3v10<4, 0, 1, (1 << 25), 3 | 8>(); d.name = "v10.wpxr1"; return d; }
      if (strcmp(force, "v10.wp") == 0) { d = variant3v10<4, 0, 0, (1 << 25), 3>(); d.name = "v10.wp"; return d; }
      if (strcmp(force, "v10.wx") == 0) { d = variant3v10<4, 0, 0, 0, 3 | 8>(); d.name = "v10.wx"; return d; }
      if (strcmp(force, "v10.wphx") == 0) { d = variant3v10<4, 0, 0, (1 << 26), 3 | 8>(); d.name = "v10.wphx"; return d; }
      if (strcmp(force, "v10.wpxs") == 0) { d = variant3v10<4, 0, 0, (1 << 25), 3 | 8 | 32>(); d.name = "v10.wpxs"; return d; }
      if (strcmp(force, "v10.wpxf1") == 0) { d = variant3v10<4, 0, 0, (1 << 25), 3 | 8 | 64>(); d.name = "v10.wpxf1"; return d; }
      if (strcmp(force, "v10.wpxf2") == 0) { d = variant3v10<4, 0, 0, (1 << 25), 3 | 8 | 128>(); d.name = "v10.wpxf2"; return d; }
      if (strcmp(force, "v10.wpxf3") == 0) { d = variant3v10<4, 0, 0, (1 << 25), 3 | 8 | 192>(); d.name = "v10.wpxf3"; return d; }
      if (strcmp(force, "v10.wpxk1f") == 0) { d = variant3v10<4, 0, 0, (1 << 25), 3 | 8 | 256>(); d.name = "v10.wpxk1f"; return d; }
      if (strcmp(force, "v10.wpxk2f") == 0) { d = variant3v10<4, 0, 0, (1 << 25), 3 | 8 | 512>(); d.name = "v10.wpxk2f"; return d; }
      if (strcmp(force, "v10.wpxk3f") == 0) { d = variant3v10<4, 0, 0, (1 << 25), 3 | 8 | 768>(); d.name = "v10.wpxk3f"; return d; }
      if (strcmp(force, "v10.wpxu") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | 128, 3 | 8>(); d.name = "v10.wpxu"; return d; }
      if (strcmp(force, "v10.wpxn") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | 2048, 3 | 8>(); d.name = "v10.wpxn"; return d; }
      if (strcmp(force, "v10.wpxb2") == 0) { d = variant3v10<4, 0, 0, (1 << 25), 3 | 8 | 1024>(); d.name = "v10.wpxb2"; return d; }
      if (strcmp(force, "v10.wpxbulk") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | 1, 3 | 8>(); d.name = "v10.wpxbulk"; return d; }
      if (strcmp(force, "v10.wpxlate") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | 2, 3 | 8>(); d.name = "v10.wpxlate"; return d; }
      if (strcmp(force, "v10.wpxv16") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | 16, 3 | 8>(); d.name = "v10.wpxv16"; return d; }
      if (strcmp(force, "v10.wpxspread") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | 64, 3 | 8>(); d.name = "v10.wpxspread"; return d; }
      if (strcmp(force, "v10.wpxbal") == 0) { d = variant3v10<4, 0, 0, (1 << 25) | 4, 3 | 8>(); d.name = "v10.wpxbal"; return d; }
      if (strcmp(force, "v10.d2") == 0) { d = variant3v10<4, 2>(); d.name = "v10.d2"; return d; }
      if (strcmp(force, "v5.r2") == 0) { d = variant3v5<4, 0, 2>(); d.name = "v5.r2"; return d; }
      if (strcmp(force, "v5.r1d1") == 0) { d = variant3v5<4, 1, 1>(); d.name = "v5.r1d1"; return d; }
      if (strcmp(force, "v5.r2d1") == 0) { d = variant3v5<4, 1, 2>(); d.name = "v5.r2d1"; return d; }
    }
#endif
  }
  return c[0];
}

// Debug: F_z = A_z B^T from S(q) (kernel 7 of the paper); one CTA per zone.
template <int D>
__global__ void kbd_form_Fz(const double *Sq, const double *tab, int k, int64_t Z, double *Fz) {
  const int n = 2 * k, p = k + 1, t = k;
  const int nk = D == 3 ? p * p * p : p * p, nt = D == 3 ? t * t * t : t * t, nq = D == 3 ? n * n * n : n * n;
  const double *B = tab, *G = tab + n * p, *Phi = tab + 2 * n * p;
  const int64_t z = blockIdx.x;
  if (z >= Z) return;
  for (int i = threadIdx.x; i < D * nk * nt; i += blockDim.x) {
    const int row = i / nt, j = i - row * nt;
    const int c = row / nk, a = row - c * nk;
    int ai[3] = {a % p, (a / p) % p, a / (p * p)};
    int ji[3] = {j % t, (j / t) % t, j / (t * t)};
    double s = 0.0;
    for (int q = 0; q < nq; ++q) {
      int qi[3] = {q % n, (q / n) % n, q / (n * n)};
      double phi = 1.0;
      for (int d = 0; d < D; ++d) phi *= Phi[qi[d] * t + ji[d]];
      double acc = 0.0;
      for (int d = 0; d < D; ++d) {
        double dw = 1.0;
        for (int e = 0; e < D; ++e) dw *= (e == d ? G : B)[qi[e] * p + ai[e]];
        acc += Sq[(z * nq + q) * D * D + c * D + d] * dw;
      }
      s += acc * phi;
    }
    Fz[(z * D * nk + row) * nt + j] = s;
  }
}

// J0^{-1} at every quadrature point of a (non-affine) initial mesh, and alpha_q det J0(q) for its volume:
// J0(q)_{cd} = sum_a x0_c(node_a) dW_a/dxi_d(q) with the tensor-product Lagrange tables of this order
// (the a1 geometry step of SURVEY §8(a), on x0; reading R19).  One thread per (zone, point); dense over
// the Nk nodes (a create-time cost, like the paper's per-run setup).
template <int D>
__global__ void kb0_point_j0inv(const double *x0, const int32_t *zn, const double *tab, int k, int64_t Z, int64_t nn,
                                double *J0inv_q, double *wdet) {
  const int n = 2 * k, p = k + 1;
  const int nq = D == 3 ? n * n * n : n * n, nk = D == 3 ? p * p * p : p * p;
  const double *B = tab, *G = tab + n * p, *w = tab + 2 * n * p + n * k;
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= Z * nq) return;
  const int64_t z = idx / nq;
  const int q = (int)(idx - z * nq);
  const int qi[3] = {q % n, (q / n) % n, q / (n * n)};
  double J[D][D];
  for (int c = 0; c < D; ++c)
    for (int d = 0; d < D; ++d) J[c][d] = 0.0;
  for (int a = 0; a < nk; ++a) {
    const int ai[3] = {a % p, (a / p) % p, a / (p * p)};
    const int64_t node = zn[z * nk + a];
    double g[D];
    for (int d = 0; d < D; ++d) {
      double f = 1.0;
      for (int t = 0; t < D; ++t) f *= (t == d ? G : B)[qi[t] * p + ai[t]];
      g[d] = f;
    }
    for (int c = 0; c < D; ++c) {
      const double xc = x0[c * nn + node];
      for (int d = 0; d < D; ++d) J[c][d] = fma(xc, g[d], J[c][d]);
    }
  }
  double alpha = 1.0;
  for (int t = 0; t < D; ++t) alpha *= w[qi[t]];
  double *o = J0inv_q + idx * D * D;
  if (D == 2) {
    const double det = J[0][0] * J[1][1] - J[0][1] * J[1][0], id = 1.0 / det;
    o[0] = J[1][1] * id; o[1] = -J[0][1] * id; o[2] = -J[1][0] * id; o[3] = J[0][0] * id;
    wdet[idx] = alpha * det;
  } else {
    const double c00 = J[1][1] * J[2][2] - J[1][2] * J[2][1], c01 = J[0][2] * J[2][1] - J[0][1] * J[2][2],
                 c02 = J[0][1] * J[1][2] - J[0][2] * J[1][1], c10 = J[1][2] * J[2][0] - J[1][0] * J[2][2],
                 c11 = J[0][0] * J[2][2] - J[0][2] * J[2][0], c12 = J[0][2] * J[1][0] - J[0][0] * J[1][2],
                 c20 = J[1][0] * J[2][1] - J[1][1] * J[2][0], c21 = J[0][1] * J[2][0] - J[0][0] * J[2][1],
                 c22 = J[0][0] * J[1][1] - J[0][1] * J[1][0];
    const double det = J[0][0] * c00 + J[0][1] * c10 + J[0][2] * c20, id = 1.0 / det;
    o[0] = c00 * id; o[1] = c01 * id; o[2] = c02 * id;
    o[3] = c10 * id; o[4] = c11 * id; o[5] = c12 * id;
    o[6] = c20 * id; o[7] = c21 * id; o[8] = c22 * id;
    wdet[idx] = alpha * det;
  }
}

}  // namespace


// ------------------------------------------------------------------------------------------------
// exchange (exchange.cuh) — out-of-line parts that report errors through fail()
// ------------------------------------------------------------------------------------------------
namespace blastcf {

int nccl_fail(ncclResult_t r, const char *what) {
  NcclApi *api = nccl_api();
  return fail(BLAST_CF_ENCCL, "%s: %s", what, api && api->GetErrorString ? api->GetErrorString(r) : "NCCL error");
}

#define NCCL_TRY(expr, what)                       \
  do {                                             \
    ncclResult_t r_ = (expr);                      \
    if (r_ != ncclSuccess) return nccl_fail(r_, what); \
  } while (0)

int nccl_get_unique_id(void *out) {
  NcclApi *api = nccl_api();
  if (!api) return fail(BLAST_CF_ENCCL, "cannot dlopen NCCL (set BLAST_CF_NCCL_LIB)");
  NCCL_TRY(api->GetUniqueId((ncclUniqueId *)out), "ncclGetUniqueId");
  return BLAST_CF_OK;
}

int exchange_create(Exchange **out, const blast_cf_mesh *mesh, int dim, int64_t nn, cudaStream_t stream,
                    const void *uid) {
  *out = nullptr;
  NcclApi *api = uid ? nccl_api() : nullptr;   // uid NULL: loopback exchange (blast_cf_eval_loopback)
  if (uid && !api) return fail(BLAST_CF_ENCCL, "cannot dlopen NCCL (set BLAST_CF_NCCL_LIB)");
  if (mesh->num_neighbors < 0 || (mesh->num_neighbors > 0 && (!mesh->nbr_rank || !mesh->nbr_offset || !mesh->nbr_nodes)))
    return fail(BLAST_CF_EINVAL, "neighbour lists");
  for (int i = 0; i < mesh->num_neighbors; ++i) {
    if (mesh->nbr_rank[i] < 0 || mesh->nbr_rank[i] >= mesh->nranks || mesh->nbr_rank[i] == mesh->rank ||
        (i > 0 && mesh->nbr_rank[i] <= mesh->nbr_rank[i - 1]) || mesh->nbr_offset[i + 1] < mesh->nbr_offset[i])
      return fail(BLAST_CF_EINVAL, "neighbour %d: ranks must be ascending, distinct from own rank", i);
  }
  const int64_t total = mesh->num_neighbors > 0 ? mesh->nbr_offset[mesh->num_neighbors] : 0;
  for (int64_t r = 0; r < total; ++r)
    if (mesh->nbr_nodes[r] < 0 || mesh->nbr_nodes[r] >= nn) return fail(BLAST_CF_EINVAL, "nbr_nodes[%lld]", (long long)r);
  Exchange *x = new (std::nothrow) Exchange();
  if (!x) return fail(BLAST_CF_ENOMEM, "host allocation");
  x->api = api; x->rank = mesh->rank; x->nranks = mesh->nranks; x->dim = dim; x->nn = nn;
  x->num_nbr = mesh->num_neighbors; x->stream = stream; x->nrows = total;
  x->nbr_rank.assign(mesh->nbr_rank, mesh->nbr_rank + x->num_nbr);
  x->nbr_offset.assign(mesh->nbr_offset, mesh->nbr_offset + x->num_nbr + 1);
  x->h_rows.assign(mesh->nbr_nodes, mesh->nbr_nodes + total);
  ExchangePlan pl = build_plan(x->rank, x->num_nbr, mesh->nbr_rank, mesh->nbr_offset, mesh->nbr_nodes);
  x->nu = (int64_t)pl.unique_nodes.size();
  int rc;
  if ((rc = upload(&x->d_rows, mesh->nbr_nodes, (size_t)total)) ||
      (rc = upload(&x->d_unodes, pl.unique_nodes.data(), pl.unique_nodes.size())) ||
      (rc = upload(&x->d_sptr, pl.src_ptr.data(), pl.src_ptr.size())) ||
      (rc = upload(&x->d_src, pl.src.data(), pl.src.size()))) {
    exchange_destroy(x);
    return rc;
  }
  if (cudaMalloc(&x->d_send, std::max<int64_t>(total * dim, 1) * sizeof(double)) != cudaSuccess ||
      cudaMalloc(&x->d_recv, std::max<int64_t>(total * dim, 1) * sizeof(double)) != cudaSuccess ||
      cudaMalloc(&x->d_tmp, 2 * sizeof(double)) != cudaSuccess ||
      cudaMalloc(&x->d_rdt, std::max(x->num_nbr, 1) * sizeof(double)) != cudaSuccess) {
    exchange_destroy(x);
    return fail(BLAST_CF_ENOMEM, "exchange buffers");
  }
  // overlap schedule: possible when the zones touching shared nodes are exactly the prefix [0, nb)
  {
    int nk = 1;
    for (int d = 0; d < dim; ++d) nk *= mesh->order + 1;
    std::vector<char> shared((size_t)std::max<int64_t>(nn, 1), 0);
    for (int64_t r = 0; r < total; ++r) shared[mesh->nbr_nodes[r]] = 1;
    int64_t nb = 0;
    bool prefix = true;
    for (int64_t z = 0; z < mesh->num_zones; ++z) {
      bool b = false;
      for (int a = 0; a < nk && !b; ++a) b = shared[mesh->zone_nodes[z * nk + a]] != 0;
      if (b) {
        if (nb != z) prefix = false;
        ++nb;
      }
    }
    const char *ov = getenv("BLAST_CF_OVERLAP");
    x->nb = nb;
    x->overlap = prefix && nb > 0 && nb < mesh->num_zones && !(ov && ov[0] == '0');
  }
  {
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);   // hi = greatest priority (numerically lowest)
    if (cudaStreamCreateWithPriority(&x->s_comm, cudaStreamNonBlocking, hi) != cudaSuccess ||
        cudaEventCreateWithFlags(&x->ev_s, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&x->ev_b, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&x->ev_i, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&x->ev_p, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&x->ev_x, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreate(&x->ev_sent) != cudaSuccess) {
      exchange_destroy(x);
      return fail(BLAST_CF_ECUDA, "exchange stream / events");
    }
  }
  if (!uid) {
    *out = x;
    return BLAST_CF_OK;
  }
  ncclUniqueId id;
  memcpy(&id, uid, sizeof id);
  ncclResult_t r = api->CommInitRank(&x->comm, x->nranks, id, x->rank);
  if (r != ncclSuccess) {
    x->comm = nullptr;
    exchange_destroy(x);
    return nccl_fail(r, "ncclCommInitRank");
  }
  *out = x;
  return BLAST_CF_OK;
}

int exchange_allreduce_sum2(Exchange *x, double *a, double *b) {
  double hv[2] = {*a, *b};
  // copies ordered on the NCCL stream (a pageable cudaMemcpy may return before its DMA lands)
  CUDA_TRY(cudaMemcpyAsync(x->d_tmp, hv, sizeof hv, cudaMemcpyHostToDevice, x->stream));
  NCCL_TRY(x->api->AllReduce(x->d_tmp, x->d_tmp, 2, ncclDouble, ncclSum, x->comm, x->stream), "ncclAllReduce(sum)");
  CUDA_TRY(cudaMemcpyAsync(hv, x->d_tmp, sizeof hv, cudaMemcpyDeviceToHost, x->stream));
  CUDA_TRY(cudaStreamSynchronize(x->stream));
  *a = hv[0];
  *b = hv[1];
  return BLAST_CF_OK;
}

void exchange_pack(Exchange *x, const double *F1) {
  if (x->nrows > 0) {
    const int blocks = (int)std::min<int64_t>((x->nrows + 255) / 256, 1184);
    xch_pack<<<blocks, 256, 0, x->stream>>>(F1, x->nn, x->dim, x->d_rows, x->nrows, x->d_send);
  }
}

void exchange_combine(Exchange *x, double *F1) {
  if (x->nu > 0) {
    const int blocks = (int)std::min<int64_t>((x->nu + 255) / 256, 1184);
    xch_combine<<<blocks, 256, 0, x->stream>>>(F1, x->nn, x->dim, x->d_unodes, x->nu, x->d_sptr, x->d_src, x->d_send,
                                               x->d_recv);
  }
}

// grouped ncclSend / ncclRecv of every neighbour's shared rows on stream st; with_dt: each rank's dt (one
// double) travels in the same group (the single-round schedule's piggy-backed min dt)
int exchange_send_rows(Exchange *x, cudaStream_t st, bool with_dt, const double *dt) {
  const int dim = x->dim;
  NCCL_TRY(x->api->GroupStart(), "ncclGroupStart");
  for (int i = 0; i < x->num_nbr; ++i) {
    const int64_t o = x->nbr_offset[i], cnt = x->nbr_offset[i + 1] - o;
    if (cnt > 0) {
      NCCL_TRY(x->api->Send(x->d_send + o * dim, (size_t)cnt * dim, ncclDouble, x->nbr_rank[i], x->comm, st), "ncclSend");
      NCCL_TRY(x->api->Recv(x->d_recv + o * dim, (size_t)cnt * dim, ncclDouble, x->nbr_rank[i], x->comm, st), "ncclRecv");
    }
    if (with_dt) {
      NCCL_TRY(x->api->Send(dt, 1, ncclDouble, x->nbr_rank[i], x->comm, st), "ncclSend(dt)");
      NCCL_TRY(x->api->Recv(x->d_rdt + i, 1, ncclDouble, x->nbr_rank[i], x->comm, st), "ncclRecv(dt)");
    }
  }
  NCCL_TRY(x->api->GroupEnd(), "ncclGroupEnd");
  return BLAST_CF_OK;
}

// single-round schedule, after KB2 (F1 = this rank's partial F.1, dt = its local min dt)
int exchange_run(Exchange *x, double *F1, double *dt) {
  if (!x->comm) return BLAST_CF_OK;   // loopback: blast_cf_eval_loopback moves the data
  exchange_pack(x, F1);
  const bool all_nbrs = x->dt_piggy;   // every rank neighbours every other (agreed by all ranks at create)
  int rc = exchange_send_rows(x, x->stream, all_nbrs, dt);
  if (rc) return rc;
  if (all_nbrs) {
    if (x->num_nbr > 0) xch_dt_combine<<<1, 32, 0, x->stream>>>(dt, x->d_rdt, x->num_nbr);
  } else {
    NCCL_TRY(x->api->AllReduce(dt, dt, 1, ncclDouble, ncclMin, x->comm, x->stream), "ncclAllReduce(min dt)");
  }
  exchange_combine(x, F1);
  return BLAST_CF_OK;
}

}  // namespace blastcf

struct blast_cf {
  int dim = 0, k = 0, nk = 0, nt = 0, nq = 0;
  int64_t Z = 0, nn = 0;
  blast_cf_params params{};
  double h0 = 0.0;
  cudaStream_t stream = nullptr;
  int device = 0;
  KB1Variant var{};
  int ncta = 0, regs = 0, local_bytes = 0, sms = 148;
  int64_t ncta_cap = 0;
  // device memory
  double *d_tab = nullptr, *d_J0inv = nullptr, *d_gamma = nullptr, *d_Fz1 = nullptr, *d_ctadt = nullptr;
  double *d_J0inv_q = nullptr;   // [Z][Nq][dim^2]: non-affine initial mesh with viscosity on (reading R19)
  bool rho_resident = false;     // blast_cf_set_rho0detJ0_host has filled the staging copy of rho0|J0|
  int32_t *d_zone_nodes = nullptr, *d_ptr = nullptr, *d_ent = nullptr;
  // host-eval staging (blast_cf_eval_host): device copies of the inputs/outputs and the zone-chunk pipeline
  double *d_in = nullptr, *d_out = nullptr;
  struct HostPipe {
    static constexpr int MAXC = 16;
    const void *plan_for = nullptr;          // KB1 function the plan was built for (autotune may switch it)
    int nch = 0;                             // zone chunks (1 = no pipelining)
    int64_t z0[MAXC + 1] = {};               // chunk c = zones [z0[c], z0[c+1])
    int64_t hi[MAXC] = {};                   // max node id over the zones of chunks 0..c (prefix max)
    int64_t lo[MAXC + 1] = {};               // min node id over the zones of chunks c..nch-1 (suffix min; lo[nch] = nn):
                                             // F.1 of nodes below lo[c+1] is final once chunks 0..c are done
    int grid[MAXC] = {}, off[MAXC] = {}, nslots = 0;   // KB1 grid and per-CTA dt slots of each chunk
    double *d_ctadt = nullptr;
    cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
    cudaEvent_t ev_in[MAXC] = {}, ev_kb1[MAXC] = {}, ev_d2h = nullptr, ev_start = nullptr;
  } hp;
  long long *d_prof = nullptr;   // stage timestamps (BLAST_CF_PROFILE=1)
  // timing
  bool timing = false;
  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  // multi-GPU
  blastcf::Exchange *xch = nullptr;
};

namespace {

void free_handle(blast_cf *h) {
  if (!h) return;
  cudaFree(h->d_tab); cudaFree(h->d_J0inv); cudaFree(h->d_J0inv_q); cudaFree(h->d_gamma); cudaFree(h->d_Fz1); cudaFree(h->d_ctadt);
  cudaFree(h->d_zone_nodes); cudaFree(h->d_ptr); cudaFree(h->d_ent); cudaFree(h->d_in); cudaFree(h->d_out); cudaFree(h->d_prof);
  for (auto &e : h->ev)
    if (e) cudaEventDestroy(e);
  if (h->xch) blastcf::exchange_destroy(h->xch);
  cudaFree(h->hp.d_ctadt);
  for (int c = 0; c < blast_cf::HostPipe::MAXC; ++c) {
    if (h->hp.ev_in[c]) cudaEventDestroy(h->hp.ev_in[c]);
    if (h->hp.ev_kb1[c]) cudaEventDestroy(h->hp.ev_kb1[c]);
  }
  if (h->hp.ev_d2h) cudaEventDestroy(h->hp.ev_d2h);
  if (h->hp.ev_start) cudaEventDestroy(h->hp.ev_start);
  if (h->hp.s_h2d) cudaStreamDestroy(h->hp.s_h2d);
  if (h->hp.s_d2h) cudaStreamDestroy(h->hp.s_d2h);
  delete h;
}


// make `v` the handle's KB1: shared-memory opt-in, register / local-memory info, grid size
int apply_variant(blast_cf *h, const KB1Variant &v) {
  if (cudaFuncSetAttribute(v.func, cudaFuncAttributeMaxDynamicSharedMemorySize, v.smem) != cudaSuccess)
    return fail(BLAST_CF_ECUDA, "cudaFuncSetAttribute(smem=%d): %s", v.smem, cudaGetErrorString(cudaGetLastError()));
  cudaFuncAttributes fa;
  if (cudaFuncGetAttributes(&fa, v.func) == cudaSuccess) {
    h->regs = fa.numRegs;
    h->local_bytes = (int)fa.localSizeBytes;
  }
  h->var = v;
  cudaDeviceGetAttribute(&h->sms, cudaDevAttrMultiProcessorCount, h->device);
  h->ncta = (int)((h->Z + v.zpc - 1) / v.zpc);
  if (v.persistent && h->ncta > 0) {
    int occ = 0, sms = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, v.func, v.nth, v.smem);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, h->device);
    h->ncta = std::min<int>(h->ncta, std::max(1, occ) * std::max(1, sms));
  }
  return BLAST_CF_OK;
}

int check_async(blast_cf *h) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(BLAST_CF_ECUDA, "CUDA error: %s", cudaGetErrorString(e));
  (void)h;
  return BLAST_CF_OK;
}

// Algorithmic flops per zone: SURVEY §8(d4)'s F_sf verbatim (the contract's model):
//   3D: 9 (4 n p^3 + 6 n^2 p^2 + 8 n^3 p) + 4 (n t^3 + n^2 t^2 + n^3 t) + 18 Nq + 500 Nq
//   2D: 6 (4 n p^2 + 4 n^2 p) + 4 (n t^2 + n^2 t) + 8 Nq + 200 Nq
// (FMA = 2 flops; c_pt = 500 / 200 per point with each div / sqrt / rsqrt = 1).  Round 1 used
// a lower model (6 n^3 p in the last stage, c_pt 420 / 160): flops_per_zone_alg below, still reported.
double flops_per_zone(int dim, int k) {
  const double n = 2 * k, p = k + 1, t = k;
  if (dim == 3)
    return 9.0 * (4 * n * p * p * p + 6 * n * n * p * p + 8 * n * n * n * p) + 4.0 * (n * t * t * t + n * n * t * t + n * n * n * t) +
           18.0 * n * n * n + 500.0 * n * n * n;
  return 6.0 * (4 * n * p * p + 4 * n * n * p) + 4.0 * (n * t * t + n * n * t) + 8.0 * n * n + 200.0 * n * n;
}
double flops_per_zone_alg(int dim, int k) {
  const double n = 2 * k, p = k + 1, t = k;
  if (dim == 3) {
    const double contr = 9.0 * (4 * n * p * p * p + 6 * n * n * p * p + 6 * n * n * n * p) +
                         4.0 * (n * t * t * t + n * n * t * t + n * n * n * t) + 2.0 * 9 * n * n * n;
    return contr + 420.0 * n * n * n;
  }
  const double contr = 6.0 * (4 * n * p * p + 4 * n * n * p) + 4.0 * (n * t * t + n * n * t) + 2.0 * 4 * n * n;
  return contr + 160.0 * n * n;
}

}  // namespace

extern "C" {

const char *blast_cf_last_error(void) { return g_last_error.c_str(); }

const char *blast_cf_error_string(int code) {
  switch (code) {
    case BLAST_CF_OK: return "BLAST_CF_OK";
    case BLAST_CF_EINVAL: return "BLAST_CF_EINVAL: invalid argument";
    case BLAST_CF_EUNSUPPORTED: return "BLAST_CF_EUNSUPPORTED: unsupported configuration";
    case BLAST_CF_ENOMEM: return "BLAST_CF_ENOMEM: out of memory";
    case BLAST_CF_ECUDA: return "BLAST_CF_ECUDA: CUDA error";
    case BLAST_CF_ENCCL: return "BLAST_CF_ENCCL: NCCL error";
  }
  return "BLAST_CF_E?: unknown error code";
}

void blast_cf_default_params(blast_cf_params *p) {
  if (!p) return;
  p->cfl = 0.5;
  p->q_quad = 2.0;
  p->q_lin = 0.5;
  p->eps_switch = 1e-12;
  p->h0 = 0.0;
  p->use_viscosity = 1;
  p->use_vorticity = 1;
}

int blast_cf_create(const blast_cf_mesh *mesh, int order, int dim, const blast_cf_params *params,
                    void *cuda_stream, const void *nccl_unique_id, blast_cf **out) {
  NvtxRange nv("blast_cf_create");
  if (!out) return fail(BLAST_CF_EINVAL, "out is NULL");
  *out = nullptr;
  if (!mesh) return fail(BLAST_CF_EINVAL, "mesh is NULL");
  if (mesh->dim != dim || mesh->order != order)
    return fail(BLAST_CF_EINVAL, "mesh dim/order (%d,%d) != arguments (%d,%d)", mesh->dim, mesh->order, dim, order);
  if (dim != 2 && dim != 3) return fail(BLAST_CF_EUNSUPPORTED, "dim %d not in {2,3}", dim);
  if (order < 1 || order > 8) return fail(BLAST_CF_EUNSUPPORTED, "order %d not in [1,8]", order);
  if (mesh->num_zones < 0 || mesh->num_nodes < 0) return fail(BLAST_CF_EINVAL, "negative sizes");
  if (mesh->num_zones > 0 && (!mesh->zone_nodes || !mesh->x0)) return fail(BLAST_CF_EINVAL, "zone_nodes/x0 NULL");
  if (!mesh->mat_gamma || mesh->num_mats < 1) return fail(BLAST_CF_EINVAL, "mat_gamma/num_mats");
  const int nranks = mesh->nranks < 1 ? 1 : mesh->nranks;
  if (nranks > 1 && !nccl_unique_id && !(params && params->h0 > 0.0))
    return fail(BLAST_CF_EINVAL, "nranks > 1 without nccl_unique_id (loopback) needs params->h0 > 0");

  blast_cf *h = new (std::nothrow) blast_cf();
  if (!h) return fail(BLAST_CF_ENOMEM, "host allocation");
  h->dim = dim; h->k = order;
  int nk = 1, nt = 1, nq = 1;
  for (int i = 0; i < dim; ++i) { nk *= order + 1; nt *= order; nq *= 2 * order; }
  h->nk = nk; h->nt = nt; h->nq = nq;
  h->Z = mesh->num_zones; h->nn = mesh->num_nodes;
  if (params) h->params = *params; else blast_cf_default_params(&h->params);
  h->stream = (cudaStream_t)cuda_stream;
  int rc = BLAST_CF_OK;
  auto bail = [&](int code) { free_handle(h); return code; };
  if (cudaGetDevice(&h->device) != cudaSuccess) return bail(fail(BLAST_CF_ECUDA, "no CUDA device"));

  // ---- validate the map ----
  const int64_t Z = h->Z, nn = h->nn;
  for (int64_t i = 0; i < Z * nk; ++i) {
    const int32_t nd = mesh->zone_nodes[i];
    if (nd < 0 || nd >= nn) return bail(fail(BLAST_CF_EINVAL, "zone_nodes[%lld] = %d out of range", (long long)i, nd));
  }
  std::vector<double> zgam(Z);
  for (int64_t z = 0; z < Z; ++z) {
    const int m = mesh->zone_mat ? mesh->zone_mat[z] : 0;
    if (m < 0 || m >= mesh->num_mats) return bail(fail(BLAST_CF_EINVAL, "zone_mat[%lld] = %d", (long long)z, m));
    zgam[z] = mesh->mat_gamma[m];
  }

  // ---- tables ----
  const blastcf::Tables1D T = blastcf::build_tables(order);
  const int p = T.p;
  std::vector<double> tab;
  tab.insert(tab.end(), T.B.begin(), T.B.end());
  tab.insert(tab.end(), T.G.begin(), T.G.end());
  tab.insert(tab.end(), T.Phi.begin(), T.Phi.end());
  tab.insert(tab.end(), T.qwt.begin(), T.qwt.end());

  // ---- per-zone J0^{-1} of the affine initial zones and the volume ----
  std::vector<double> J0inv((size_t)Z * dim * dim);
  long double vol = 0.0L;
  bool affine = true;
  for (int64_t z = 0; z < Z; ++z) {
    const int32_t *zn = mesh->zone_nodes + z * nk;
    long double J[3][3] = {{0}}, X0[3];
    for (int c = 0; c < dim; ++c) X0[c] = mesh->x0[c * nn + zn[0]];
    for (int d = 0; d < dim; ++d) {
      int a = (d == 0 ? order : d == 1 ? order * p : order * p * p);   // vertex with l_d = k
      for (int c = 0; c < dim; ++c) J[c][d] = (long double)mesh->x0[c * nn + zn[a]] - X0[c];
    }
    // affinity: x_a = x_0 + J xi_a for every node a
    long double scale = 0.0L;
    for (int c = 0; c < dim; ++c)
      for (int d = 0; d < dim; ++d) scale = std::max(scale, fabsl(J[c][d]));
    for (int a = 0; a < nk && affine; ++a) {
      const int li[3] = {a % p, (a / p) % p, a / (p * p)};
      for (int c = 0; c < dim; ++c) {
        long double xa = X0[c];
        for (int d = 0; d < dim; ++d) xa += J[c][d] * (long double)T.gll[li[d]];
        if (fabsl(xa - (long double)mesh->x0[c * nn + zn[a]]) > 1e-11L * scale) { affine = false; }
      }
    }
    long double det, inv[3][3];
    if (dim == 2) {
      det = J[0][0] * J[1][1] - J[0][1] * J[1][0];
      inv[0][0] = J[1][1] / det; inv[0][1] = -J[0][1] / det;
      inv[1][0] = -J[1][0] / det; inv[1][1] = J[0][0] / det;
    } else {
      const long double c00 = J[1][1] * J[2][2] - J[1][2] * J[2][1], c01 = J[0][2] * J[2][1] - J[0][1] * J[2][2],
                        c02 = J[0][1] * J[1][2] - J[0][2] * J[1][1], c10 = J[1][2] * J[2][0] - J[1][0] * J[2][2],
                        c11 = J[0][0] * J[2][2] - J[0][2] * J[2][0], c12 = J[0][2] * J[1][0] - J[0][0] * J[1][2],
                        c20 = J[1][0] * J[2][1] - J[1][1] * J[2][0], c21 = J[0][1] * J[2][0] - J[0][0] * J[2][1],
                        c22 = J[0][0] * J[1][1] - J[0][1] * J[1][0];
      det = J[0][0] * c00 + J[0][1] * c10 + J[0][2] * c20;
      inv[0][0] = c00 / det; inv[0][1] = c01 / det; inv[0][2] = c02 / det;
      inv[1][0] = c10 / det; inv[1][1] = c11 / det; inv[1][2] = c12 / det;
      inv[2][0] = c20 / det; inv[2][1] = c21 / det; inv[2][2] = c22 / det;
    }
    vol += det;
    for (int c = 0; c < dim; ++c)
      for (int d = 0; d < dim; ++d) J0inv[(size_t)z * dim * dim + c * dim + d] = (double)inv[c][d];
  }
  const bool point_j0 = !affine && h->params.use_viscosity;   // reading R19: J0^{-1} at every point
  if (!affine) {   // the mesh volume by quadrature (the vertex-difference det above is exact only for affine zones)
    const int64_t npts = Z * nq;
    double *dx0 = nullptr, *dtab = nullptr, *dw = nullptr;
    int32_t *dzn = nullptr;
    std::vector<double> w((size_t)std::max<int64_t>(npts, 1));
    int rc2 = BLAST_CF_OK;
    if ((rc2 = upload(&dx0, mesh->x0, (size_t)dim * nn)) || (rc2 = upload(&dtab, tab.data(), tab.size())) ||
        (rc2 = upload(&dzn, mesh->zone_nodes, (size_t)Z * nk))) {
      cudaFree(dx0); cudaFree(dtab); cudaFree(dzn);
      return bail(rc2);
    }
    if (cudaMalloc(&h->d_J0inv_q, std::max<int64_t>(npts, 1) * dim * dim * sizeof(double)) != cudaSuccess ||
        cudaMalloc(&dw, std::max<int64_t>(npts, 1) * sizeof(double)) != cudaSuccess) {
      cudaFree(dx0); cudaFree(dtab); cudaFree(dzn); cudaFree(dw);
      return bail(fail(BLAST_CF_ENOMEM, "per-point J0 buffer (%lld points)", (long long)npts));
    }
    if (npts > 0) {
      const unsigned blocks = (unsigned)((npts + 127) / 128);
      if (dim == 3) kb0_point_j0inv<3><<<blocks, 128>>>(dx0, dzn, dtab, order, Z, nn, h->d_J0inv_q, dw);
      else kb0_point_j0inv<2><<<blocks, 128>>>(dx0, dzn, dtab, order, Z, nn, h->d_J0inv_q, dw);
    }
    const cudaError_t ce = npts > 0 ? cudaMemcpy(w.data(), dw, npts * sizeof(double), cudaMemcpyDeviceToHost) : cudaSuccess;
    cudaFree(dx0); cudaFree(dtab); cudaFree(dzn); cudaFree(dw);
    if (ce != cudaSuccess) return bail(fail(BLAST_CF_ECUDA, "per-point J0 kernel: %s", cudaGetErrorString(ce)));
    vol = 0.0L;
    for (int64_t i = 0; i < npts; ++i) vol += (long double)w[i];
    if (!point_j0) { cudaFree(h->d_J0inv_q); h->d_J0inv_q = nullptr; }
  }

  // ---- multi-GPU: communicator, global volume / zone count for h0 ----
  double gvol = (double)vol, gz = (double)Z;
  if (nranks > 1) {
    rc = blastcf::exchange_create(&h->xch, mesh, dim, nn, h->stream, nccl_unique_id);
    if (rc) { free_handle(h); return rc; }
    if (nccl_unique_id) {
      rc = blastcf::exchange_allreduce_sum2(h->xch, &gvol, &gz);
      if (rc) { free_handle(h); return rc; }
      // the schedule must be the same on every rank (NCCL calls are matched in order): overlap only if every
      // rank can, the piggy-backed dt only if every rank neighbours every other
      double no_overlap = h->xch->overlap ? 0.0 : 1.0, not_all = h->xch->num_nbr == nranks - 1 ? 0.0 : 1.0;
      rc = blastcf::exchange_allreduce_sum2(h->xch, &no_overlap, &not_all);
      if (rc) { free_handle(h); return rc; }
      h->xch->overlap = h->xch->overlap && no_overlap == 0.0;
      h->xch->dt_piggy = not_all == 0.0;
    } else {
      h->xch->dt_piggy = h->xch->num_nbr == nranks - 1;   // loopback: blast_cf_eval_loopback decides per group
    }
  }
  h->h0 = h->params.h0 > 0.0 ? h->params.h0 : pow(gvol / gz, 1.0 / dim) / order;

  // ---- inverse map: node -> entries z*dim*nk + a in ascending zone id ----
  std::vector<int32_t> ptr(nn + 1, 0), ent((size_t)Z * nk);
  if ((double)Z * dim * nk >= 2147483647.0) return bail(fail(BLAST_CF_EUNSUPPORTED, "too many zones for int32 entries"));
  for (int64_t i = 0; i < Z * nk; ++i) ptr[mesh->zone_nodes[i] + 1]++;
  for (int64_t i = 0; i < nn; ++i) ptr[i + 1] += ptr[i];
  {
    std::vector<int32_t> fill(ptr.begin(), ptr.end() - 1);
    for (int64_t z = 0; z < Z; ++z)
      for (int a = 0; a < nk; ++a) ent[fill[mesh->zone_nodes[z * nk + a]]++] = (int32_t)(z * dim * nk + a);
  }

  // ---- constant tables: 1-D tables of this order, eigen-root polynomial (identical for every handle) ----
  if (cudaMemcpyToSymbol(c_tabs, tab.data(), tab.size() * sizeof(double), ctab_off(order) * sizeof(double)) !=
      cudaSuccess)
    return bail(fail(BLAST_CF_ECUDA, "cudaMemcpyToSymbol(c_tabs)"));
  {
    const std::vector<double> ep = blastcf::eig_root_poly(EIG_POLY_DEG);
    if (cudaMemcpyToSymbol(c_eig_poly, ep.data(), ep.size() * sizeof(double)) != cudaSuccess)
      return bail(fail(BLAST_CF_ECUDA, "cudaMemcpyToSymbol(c_eig_poly)"));
  }

  // ---- kernel variant ----
  h->var = select_variant(dim, order, point_j0);
  if (!h->var.launch) return bail(fail(BLAST_CF_EUNSUPPORTED, "no kernel for dim %d order %d", dim, order));
  if ((rc = apply_variant(h, h->var))) return bail(rc);
  for (const KB1Variant &c : kb1_usable(dim, order, point_j0))   // per-CTA dt slots for any candidate
    h->ncta_cap = std::max<int64_t>(h->ncta_cap, (Z + c.zpc - 1) / c.zpc);

  // ---- uploads ----
  if ((rc = upload(&h->d_tab, tab.data(), tab.size())) ||
      (rc = upload(&h->d_J0inv, J0inv.data(), J0inv.size())) ||
      (rc = upload(&h->d_gamma, zgam.data(), zgam.size())) ||
      (rc = upload(&h->d_zone_nodes, mesh->zone_nodes, (size_t)Z * nk)) ||
      (rc = upload(&h->d_ptr, ptr.data(), ptr.size())) || (rc = upload(&h->d_ent, ent.data(), ent.size())))
    return bail(rc);
  if (cudaMalloc(&h->d_Fz1, std::max<size_t>((size_t)Z * dim * nk, 1) * sizeof(double)) != cudaSuccess ||
      cudaMalloc(&h->d_ctadt, (std::max<int64_t>(h->ncta_cap, 1) + 2) * sizeof(double)) != cudaSuccess)
    return bail(fail(BLAST_CF_ENOMEM, "workspace allocation"));
  for (auto &e : h->ev)
    if (cudaEventCreate(&e) != cudaSuccess) return bail(fail(BLAST_CF_ECUDA, "event create"));
  if (getenv("BLAST_CF_PROFILE") && cudaMalloc(&h->d_prof, std::max<int64_t>(h->ncta_cap, 1) * 16 * sizeof(long long)) != cudaSuccess)
    return bail(fail(BLAST_CF_ENOMEM, "profile buffer"));
  if (h->d_prof) cudaMemset(h->d_prof, 0, std::max<int64_t>(h->ncta_cap, 1) * 16 * sizeof(long long));
  // the uploads above are legacy-stream copies from pageable memory: make sure they have landed before any eval
  // is enqueued on a (possibly non-blocking) user stream
  if (cudaDeviceSynchronize() != cudaSuccess) return bail(fail(BLAST_CF_ECUDA, "create: %s", cudaGetErrorString(cudaGetLastError())));
  *out = h;
  return BLAST_CF_OK;
}

static KB1Args make_args(const blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                         double *out_FTv, double *Sq) {
  KB1Args a;
  a.x = x; a.v = v; a.e = e; a.rho0detJ0 = rho0detJ0;
  a.zone_nodes = h->d_zone_nodes; a.J0inv = h->d_J0inv; a.J0inv_q = h->d_J0inv_q; a.zone_gamma = h->d_gamma; a.tab = h->d_tab;
  a.Fz1 = h->d_Fz1; a.FTv = out_FTv; a.cta_dt = h->d_ctadt; a.Sq = Sq; a.prof = h->d_prof;
  a.num_zones = h->Z; a.num_nodes = h->nn; a.zero = 0;
  a.ph.cfl = h->params.cfl; a.ph.q_quad = h->params.q_quad; a.ph.q_lin = h->params.q_lin;
  a.ph.eps_sw = h->params.eps_switch; a.ph.inv_2eps = 0.5 / h->params.eps_switch; a.ph.h0 = h->h0; a.ph.k = (double)h->k;
  a.ph.use_visc = h->params.use_viscosity; a.ph.use_vort = h->params.use_vorticity;
  return a;
}

// KB1 on the zone range [z0, z0 + zc) (zone-indexed pointers shifted), per-CTA dt slots from slot_off
static void launch_range(const blast_cf *h, const KB1Args &base, int64_t z0, int64_t zc, int grid, int slot_off,
                         cudaStream_t st) {
  if (zc <= 0 || grid <= 0) return;
  KB1Args ac = base;
  const int dd = h->dim * h->dim;
  ac.zone_nodes = h->d_zone_nodes + z0 * h->nk; ac.J0inv = h->d_J0inv + z0 * dd; ac.zone_gamma = h->d_gamma + z0;
  if (base.J0inv_q) ac.J0inv_q = base.J0inv_q + z0 * h->nq * dd;
  if (base.Sq) ac.Sq = base.Sq + z0 * h->nq * dd;
  ac.e = base.e + z0 * h->nt; ac.rho0detJ0 = base.rho0detJ0 + z0 * h->nq; ac.Fz1 = h->d_Fz1 + z0 * h->dim * h->nk;
  ac.FTv = base.FTv + z0 * h->nt; ac.cta_dt = h->d_ctadt + slot_off; ac.num_zones = zc; ac.prof = nullptr;
  h->var.launch(ac, grid, st);
}

// grid of a range launch; `reserve`: persistent kernels leave that many SMs' worth of CTAs to the comm stream
static int range_grid(const blast_cf *h, int64_t zc, int reserve_sms) {
  int64_t g = (zc + h->var.zpc - 1) / h->var.zpc;
  if (h->var.persistent) {
    int cap = h->ncta;
    if (reserve_sms > 0 && h->sms > reserve_sms) cap -= (int)(((int64_t)reserve_sms * h->ncta + h->sms - 1) / h->sms);
    g = std::min<int64_t>(g, std::max(cap, 1));
  }
  return (int)g;
}

// Overlap schedule: the boundary and the interior zones run CONCURRENTLY as two launches (boundary on the
// comm stream, interior on the handle's stream); persistent kernels split the resident CTAs in proportion to
// the zone counts, so both finish together while the boundary rows' exchange runs on the SMs the boundary
// launch frees (round 2; a boundary-first sequential split paid each launch's pipeline fill twice).
static void overlap_grids(const blast_cf *h, int64_t nb, int64_t ni, int *gb, int *gi) {
  if (h->var.persistent && h->ncta >= 2) {
    const int tot = h->ncta;
    int b = (int)((double)tot * (double)nb / (double)(nb + ni) + 0.5);
    b = std::min(std::max(b, 1), tot - 1);
    *gb = (int)std::min<int64_t>(b, (nb + h->var.zpc - 1) / h->var.zpc);
    *gi = (int)std::min<int64_t>(tot - b, (ni + h->var.zpc - 1) / h->var.zpc);
  } else {
    *gb = range_grid(h, nb, 0);
    *gi = range_grid(h, ni, 0);
  }
}


// KB2 on nodes [n0, n1) (default: all); dt != nullptr: its last block also reduces the per-CTA dt slots
static void launch_kb2(const blast_cf *h, double *F1, const double *cta_dt, int ncta, double *dt, cudaStream_t st,
                       int64_t n0 = 0, int64_t n1 = -1) {
  if (n1 < 0) n1 = h->nn;
  const int gthreads = 256;
  const int64_t gblocks = std::max<int64_t>(1, (n1 - n0 + gthreads - 1) / gthreads);
  if (h->dim == 3)
    kb2_gather<3, 8><<<(unsigned)gblocks, gthreads, 0, st>>>(h->d_Fz1, h->d_ptr, h->d_ent, h->nn, n0, n1, h->nk, F1, cta_dt,
                                                             ncta, dt);
  else
    kb2_gather<2, 4><<<(unsigned)gblocks, gthreads, 0, st>>>(h->d_Fz1, h->d_ptr, h->d_ent, h->nn, n0, n1, h->nk, F1, cta_dt,
                                                             ncta, dt);
}

static void launch_pack_gather(const blast_cf *h, cudaStream_t st) {
  const blastcf::Exchange *x = h->xch;
  if (x->nrows <= 0) return;
  const int blocks = (int)std::min<int64_t>((x->nrows + 127) / 128, 1184);
  blastcf::xch_pack_gather<<<blocks, 128, 0, st>>>(h->d_Fz1, h->d_ptr, h->d_ent, h->nk, h->dim, x->d_rows, x->nrows,
                                                   x->d_send);
}

// Overlap schedule of a multi-rank NCCL handle: boundary zones, then the exchange of their
// shared rows on the comm stream while the interior zones compute; the dt allreduce overlaps KB2.
static int eval_overlap(blast_cf *h, const KB1Args &a, double *out_Fdot1, double *out_dt_min) {
  NvtxRange nv("blast_cf_eval: overlap schedule");
  blastcf::Exchange *x = h->xch;
  const int64_t nb = x->nb, ni = h->Z - nb;
  int gb = 0, gi = 0;
  overlap_grids(h, nb, ni, &gb, &gi);
  if (h->timing) cudaEventRecord(h->ev[0], h->stream);
  CUDA_TRY(cudaEventRecord(x->ev_s, h->stream));          // the inputs are ready
  CUDA_TRY(cudaStreamWaitEvent(x->s_comm, x->ev_s, 0));
  launch_range(h, a, 0, nb, gb, 0, x->s_comm);             // boundary zones (comm stream) ...
  CUDA_TRY(cudaEventRecord(x->ev_b, x->s_comm));
  launch_pack_gather(h, x->s_comm);                         // ... then their shared rows out
  int rc = blastcf::exchange_send_rows(x, x->s_comm, false, nullptr);
  if (rc) return rc;
  if (h->timing) cudaEventRecord(x->ev_sent, x->s_comm);
  launch_range(h, a, nb, ni, gi, gb, h->stream);            // interior zones, concurrently (handle's stream)
  CUDA_TRY(cudaEventRecord(x->ev_i, h->stream));
  if (h->timing) cudaEventRecord(h->ev[1], h->stream);
  CUDA_TRY(cudaStreamWaitEvent(x->s_comm, x->ev_i, 0));
  blastcf::xch_dt_reduce<<<1, 256, 0, x->s_comm>>>(h->d_ctadt, gb + gi, out_dt_min);
  if (x->api->AllReduce(out_dt_min, out_dt_min, 1, ncclDouble, ncclMin, x->comm, x->s_comm) != ncclSuccess)
    return fail(BLAST_CF_ENCCL, "ncclAllReduce(min dt)");
  CUDA_TRY(cudaEventRecord(x->ev_x, x->s_comm));
  CUDA_TRY(cudaStreamWaitEvent(h->stream, x->ev_b, 0));     // KB2 needs the boundary zones too
  launch_kb2(h, out_Fdot1, nullptr, 0, x->d_tmp, h->stream);   // node gather; dt comes from the comm stream
  if (h->timing) cudaEventRecord(h->ev[2], h->stream);
  CUDA_TRY(cudaStreamWaitEvent(h->stream, x->ev_x, 0));
  blastcf::exchange_combine(x, out_Fdot1);
  if (h->timing) cudaEventRecord(h->ev[3], h->stream);
  return check_async(h);
}

// Peer-memory transport (p2p.cuh): the shared rows are computed by the kernel that stores
// them into the neighbours' mailboxes, the dt goes to every rank's mailbox, the combine acquires both.
// Overlap schedule as eval_overlap (boundary zones on the comm stream beside the interior zones; the rows
// leave as soon as the boundary zones are done); otherwise one round after KB1 and KB2.  No NCCL call.
static int eval_p2p(blast_cf *h, const KB1Args &a, double *out_Fdot1, double *out_dt_min) {
  NvtxRange nv("blast_cf_eval: peer-memory exchange");
  blastcf::Exchange *x = h->xch;
  blastcf::P2PHost &p = x->p2p;
  const uint64_t E = ++p.epoch;
  auto send_rows = [&](cudaStream_t st) {
    if (x->num_nbr > 0)
      blastcf::p2p_send_rows<<<p.send_blocks, 256, 0, st>>>(h->d_Fz1, h->d_ptr, h->d_ent, h->nk, h->dim, x->d_rows, p.dev, E);
  };
  auto combine = [&](cudaStream_t st) {
    blastcf::p2p_combine<<<p.combine_blocks, 256, 0, st>>>(out_Fdot1, h->nn, h->dim, x->d_unodes, x->nu, x->d_sptr,
                                                          x->d_src, out_dt_min, p.dev, E);
  };
  if (h->timing) cudaEventRecord(h->ev[0], h->stream);
  if (x->overlap) {
    const int64_t nb = x->nb, ni = h->Z - nb;
    int gb = 0, gi = 0;
    overlap_grids(h, nb, ni, &gb, &gi);
    CUDA_TRY(cudaEventRecord(x->ev_s, h->stream));
    CUDA_TRY(cudaStreamWaitEvent(x->s_comm, x->ev_s, 0));
    launch_range(h, a, 0, nb, gb, 0, x->s_comm);             // boundary zones (comm stream) ...
    CUDA_TRY(cudaEventRecord(x->ev_b, x->s_comm));
    send_rows(x->s_comm);                                     // ... their rows straight into the neighbours
    if (h->timing) cudaEventRecord(x->ev_sent, x->s_comm);
    launch_range(h, a, nb, ni, gi, gb, h->stream);            // interior zones, concurrently
    CUDA_TRY(cudaEventRecord(x->ev_i, h->stream));
    if (h->timing) cudaEventRecord(h->ev[1], h->stream);
    CUDA_TRY(cudaStreamWaitEvent(x->s_comm, x->ev_i, 0));
    blastcf::p2p_send_dt<<<1, 256, 0, x->s_comm>>>(h->d_ctadt, gb + gi, out_dt_min, p.dev, E);
    CUDA_TRY(cudaEventRecord(x->ev_x, x->s_comm));
    CUDA_TRY(cudaStreamWaitEvent(h->stream, x->ev_b, 0));
    launch_kb2(h, out_Fdot1, nullptr, 0, nullptr, h->stream);
    if (h->timing) cudaEventRecord(h->ev[2], h->stream);
    CUDA_TRY(cudaStreamWaitEvent(h->stream, x->ev_x, 0));
    combine(h->stream);
  } else {
    if (h->ncta > 0) h->var.launch(a, h->ncta, h->stream);
    if (h->timing) cudaEventRecord(h->ev[1], h->stream);
    launch_kb2(h, out_Fdot1, nullptr, 0, nullptr, h->stream);
    if (h->timing) cudaEventRecord(h->ev[2], h->stream);
    send_rows(h->stream);
    blastcf::p2p_send_dt<<<1, 256, 0, h->stream>>>(h->d_ctadt, h->ncta, out_dt_min, p.dev, E);
    combine(h->stream);
  }
  if (h->timing) cudaEventRecord(h->ev[3], h->stream);
  return check_async(h);
}

static int eval_impl(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                     double *out_Fdot1, double *out_FTv, double *out_dt_min, double *Sq) {
  if (!h) return fail(BLAST_CF_EINVAL, "handle is NULL");
  if (!out_dt_min || ((!x || !v || !out_Fdot1) && h->nn > 0) || ((!e || !rho0detJ0 || !out_FTv) && h->Z > 0))
    return fail(BLAST_CF_EINVAL, "NULL array argument");
  int rc = check_async(h);
  if (rc) return rc;
  const KB1Args a = make_args(h, x, v, e, rho0detJ0, out_FTv, Sq);
  if (h->xch && h->xch->p2p.connected) return eval_p2p(h, a, out_Fdot1, out_dt_min);
  if (h->xch && h->xch->comm && h->xch->overlap) return eval_overlap(h, a, out_Fdot1, out_dt_min);
  NvtxRange nv("blast_cf_eval");
  if (h->timing) cudaEventRecord(h->ev[0], h->stream);
  if (h->ncta > 0) h->var.launch(a, h->ncta, h->stream);
  if (h->timing) cudaEventRecord(h->ev[1], h->stream);
  launch_kb2(h, out_Fdot1, h->d_ctadt, h->ncta, out_dt_min, h->stream);
  if (h->timing) cudaEventRecord(h->ev[2], h->stream);
  if (h->xch) {   // single-round schedule (a loopback handle: local part only, blast_cf_eval_loopback exchanges)
    rc = blastcf::exchange_run(h->xch, out_Fdot1, out_dt_min);
    if (rc) return rc;
  }
  if (h->timing) cudaEventRecord(h->ev[3], h->stream);
  return check_async(h);
}

}  // extern "C"

namespace blastcf {

int handle_view(const blast_cf *h, HandleView *o) {
  if (!h || !o) return fail(BLAST_CF_EINVAL, "NULL argument");
  o->dim = h->dim; o->k = h->k; o->nk = h->nk; o->nt = h->nt; o->nq = h->nq;
  o->Z = h->Z; o->nn = h->nn; o->stream = h->stream; o->device = h->device;
  o->zone_nodes = h->d_zone_nodes; o->ptr = h->d_ptr; o->ent = h->d_ent; o->tab = h->d_tab;
  o->multi_rank = h->xch != nullptr;
  o->rank = h->xch ? h->xch->rank : 0;
  o->nranks = h->xch ? h->xch->nranks : 1;
  o->loopback = h->xch != nullptr && h->xch->comm == nullptr;
  return BLAST_CF_OK;
}

int eval_with_S(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                double *out_Fdot1, double *out_FTv, double *out_dt_min, double *Sq) {
  return eval_impl(h, x, v, e, rho0detJ0, out_Fdot1, out_FTv, out_dt_min, Sq);
}

int set_error(int code, const char *msg) { return fail(code, "%s", msg); }

// a loopback group: hs[r] is rank r of an n-rank decomposition without a communicator
static int check_group(blast_cf *const *hs, int n, bool *loop) {
  if (!hs || n < 1 || !hs[0]) return fail(BLAST_CF_EINVAL, "NULL group");
  *loop = hs[0]->xch && !hs[0]->xch->comm;
  if (!*loop) return n == 1 ? BLAST_CF_OK : fail(BLAST_CF_EINVAL, "an NCCL group call drives one rank (n = 1)");
  for (int r = 0; r < n; ++r)
    if (!hs[r] || !hs[r]->xch || hs[r]->xch->comm || hs[r]->xch->p2p.connected || hs[r]->xch->nranks != n ||
        hs[r]->xch->rank != r)
      return fail(BLAST_CF_EINVAL, "handle %d is not rank %d of a %d-rank loopback group", r, r, n);
  return BLAST_CF_OK;
}

// rank r's recv rows from q are rank q's send rows for r (same order: global node id)
static int loopback_move(blast_cf *const *hs, int n) {
  for (int r = 0; r < n; ++r) CUDA_TRY(cudaStreamSynchronize(hs[r]->stream));
  for (int r = 0; r < n; ++r) {
    Exchange *xr = hs[r]->xch;
    for (int i = 0; i < xr->num_nbr; ++i) {
      const int q = xr->nbr_rank[i];
      Exchange *xq = hs[q]->xch;
      int iq = -1;
      for (int t = 0; t < xq->num_nbr; ++t)
        if (xq->nbr_rank[t] == r) iq = t;
      const int64_t cnt = xr->nbr_offset[i + 1] - xr->nbr_offset[i];
      if (iq < 0 || xq->nbr_offset[iq + 1] - xq->nbr_offset[iq] != cnt)
        return fail(BLAST_CF_EINVAL, "ranks %d and %d disagree on their shared nodes", r, q);
      CUDA_TRY(cudaMemcpyAsync(xr->d_recv + xr->nbr_offset[i] * xr->dim, xq->d_send + xq->nbr_offset[iq] * xq->dim,
                               cnt * xr->dim * sizeof(double), cudaMemcpyDeviceToDevice, hs[r]->stream));
    }
  }
  return BLAST_CF_OK;
}

int group_exchange_sum(blast_cf *const *hs, int n, double *const *vec) {
  bool loop = false;
  int rc = check_group(hs, n, &loop);
  if (rc) return rc;
  if (!hs[0]->xch) return BLAST_CF_OK;   // single rank: nothing is shared
  if (!loop) {
    Exchange *x = hs[0]->xch;
    const int dim = x->dim;
    exchange_pack(x, vec[0]);
    NCCL_TRY(x->api->GroupStart(), "ncclGroupStart");
    for (int i = 0; i < x->num_nbr; ++i) {
      const int64_t o = x->nbr_offset[i], cnt = x->nbr_offset[i + 1] - o;
      if (cnt == 0) continue;
      NCCL_TRY(x->api->Send(x->d_send + o * dim, (size_t)cnt * dim, ncclDouble, x->nbr_rank[i], x->comm, x->stream), "ncclSend");
      NCCL_TRY(x->api->Recv(x->d_recv + o * dim, (size_t)cnt * dim, ncclDouble, x->nbr_rank[i], x->comm, x->stream), "ncclRecv");
    }
    NCCL_TRY(x->api->GroupEnd(), "ncclGroupEnd");
    exchange_combine(x, vec[0]);
    return BLAST_CF_OK;
  }
  for (int r = 0; r < n; ++r) exchange_pack(hs[r]->xch, vec[r]);
  if ((rc = loopback_move(hs, n))) return rc;
  for (int r = 0; r < n; ++r) exchange_combine(hs[r]->xch, vec[r]);
  return BLAST_CF_OK;
}

int group_allreduce(blast_cf *const *hs, int n, double *const *buf, int count, int op) {
  bool loop = false;
  int rc = check_group(hs, n, &loop);
  if (rc) return rc;
  if (!hs[0]->xch || count <= 0) return BLAST_CF_OK;
  if (!loop) {
    Exchange *x = hs[0]->xch;
    const ncclRedOp_t o = op == 0 ? ncclSum : op == 1 ? ncclMin : ncclMax;
    NCCL_TRY(x->api->AllReduce(buf[0], buf[0], (size_t)count, ncclDouble, o, x->comm, x->stream), "ncclAllReduce");
    return BLAST_CF_OK;
  }
  std::vector<double> acc((size_t)count), part((size_t)count);
  for (int r = 0; r < n; ++r) {   // ascending rank order
    CUDA_TRY(cudaMemcpyAsync(part.data(), buf[r], count * sizeof(double), cudaMemcpyDeviceToHost, hs[r]->stream));
    CUDA_TRY(cudaStreamSynchronize(hs[r]->stream));
    for (int i = 0; i < count; ++i)
      acc[i] = r == 0 ? part[i] : op == 0 ? acc[i] + part[i] : op == 1 ? std::min(acc[i], part[i]) : std::max(acc[i], part[i]);
  }
  for (int r = 0; r < n; ++r) {
    CUDA_TRY(cudaMemcpyAsync(buf[r], acc.data(), count * sizeof(double), cudaMemcpyHostToDevice, hs[r]->stream));
    CUDA_TRY(cudaStreamSynchronize(hs[r]->stream));
  }
  return BLAST_CF_OK;
}

int owner_weights(const blast_cf *h, double *out) {
  if (!h->xch) {
    std::fill(out, out + h->nn, 1.0);
    return BLAST_CF_OK;
  }
  const Exchange *x = h->xch;   // a neighbour with a lower rank owns every node it shares with us
  return blast_cf_owner_mask(x->rank, x->num_nbr, x->nbr_rank.data(), x->nbr_offset.data(), x->h_rows.data(), h->nn, out);
}

}  // namespace blastcf

extern "C" {

int blast_cf_eval(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                  double *out_Fdot1, double *out_FTv, double *out_dt_min) {
  return eval_impl(h, x, v, e, rho0detJ0, out_Fdot1, out_FTv, out_dt_min, nullptr);
}

// The host-buffer entry overlaps the PCIe transfers with the corner force: the zones are split into up
// to 8 contiguous chunks; chunk c's KB1 starts as soon as its inputs are on the device (the node prefix
// [0, hi[c]] of x and v, its e and rho0|J0| slices, copied on a second stream), its F^T v slice goes back
// on a third stream while later chunks compute, and KB2 + the F.1 copy follow the last chunk.  Each chunk's
// KB1 is the same kernel on a zone sub-range (shifted zone-indexed pointers), with its own per-CTA dt slots.
static int host_plan(blast_cf *h) {
  blast_cf::HostPipe &P = h->hp;
  if (P.plan_for == h->var.func) return BLAST_CF_OK;
  // zones one wave of resident CTAs covers: the persistent grid, else occupancy x SMs
  int resident = h->ncta;
  if (!h->var.persistent) {
    int occ = 0, sms = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, h->var.func, h->var.nth, h->var.smem);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, h->device);
    resident = std::max(1, occ) * std::max(1, sms);
  }
  const int64_t per_wave = (int64_t)std::max(resident, 1) * std::max(h->var.zpc, 1);
  const char *env_ch = getenv("BLAST_CF_HOST_CHUNKS");   // default 8 (measured with the taper below)
  const int max_ch = std::min(blast_cf::HostPipe::MAXC, env_ch ? std::max(1, atoi(env_ch)) : 8);
  int nch = (int)std::min<int64_t>(max_ch, h->Z / (2 * per_wave));
  if (h->xch) nch = 1;   // multi-rank: keep the plain path (the exchange follows KB2 anyway)
  nch = std::max(nch, 1);
  std::vector<int32_t> zn((size_t)h->Z * h->nk);
  if (nch > 1) CUDA_TRY(cudaMemcpy(zn.data(), h->d_zone_nodes, zn.size() * sizeof(int32_t), cudaMemcpyDeviceToHost));
  P.nch = nch;
  P.nslots = 0;
  int64_t hi = -1;
  for (int c = 0; c < nch; ++c) {
    // chunk sizes taper linearly (weights nch + t - c, t = taper): the last chunk's corner force and copies
    // are the pipeline's exposed tail, so it is made the smallest
    const char *tp = getenv("BLAST_CF_HOST_TAPER");
    const double taper = tp ? atof(tp) : 1.5;
    auto cum = [&](int cc) {   // sum of the first cc weights / all weights
      double s_ = 0.0, t_ = 0.0;
      for (int i = 0; i < nch; ++i) {
        const double w = taper > 0.0 ? (double)(nch - i) + taper : 1.0;
        if (i < cc) s_ += w;
        t_ += w;
      }
      return s_ / t_;
    };
    P.z0[c] = c == 0 ? 0 : (int64_t)(h->Z * cum(c));
    P.z0[c + 1] = c + 1 == nch ? h->Z : (int64_t)(h->Z * cum(c + 1));
    for (size_t i = (size_t)P.z0[c] * h->nk; nch > 1 && i < (size_t)P.z0[c + 1] * h->nk; ++i) hi = std::max<int64_t>(hi, zn[i]);
    P.hi[c] = nch > 1 ? hi : h->nn - 1;
    const int64_t zc = P.z0[c + 1] - P.z0[c];
    int g = (int)((zc + h->var.zpc - 1) / h->var.zpc);
    if (h->var.persistent) g = std::min(g, h->ncta);
    P.grid[c] = g;
    P.off[c] = P.nslots;
    P.nslots += g;
  }
  P.lo[nch] = h->nn;
  for (int c = nch - 1; c >= 0; --c) {
    int64_t m = P.lo[c + 1];
    for (size_t i = (size_t)P.z0[c] * h->nk; nch > 1 && i < (size_t)P.z0[c + 1] * h->nk; ++i) m = std::min<int64_t>(m, zn[i]);
    P.lo[c] = m;
  }
  cudaFree(P.d_ctadt);
  P.d_ctadt = nullptr;
  CUDA_TRY(cudaMalloc(&P.d_ctadt, std::max(P.nslots, 1) * sizeof(double)));
  if (!P.s_h2d) {
    CUDA_TRY(cudaStreamCreateWithFlags(&P.s_h2d, cudaStreamNonBlocking));
    CUDA_TRY(cudaStreamCreateWithFlags(&P.s_d2h, cudaStreamNonBlocking));
    for (int c = 0; c < blast_cf::HostPipe::MAXC; ++c) {
      CUDA_TRY(cudaEventCreateWithFlags(&P.ev_in[c], cudaEventDisableTiming));
      CUDA_TRY(cudaEventCreateWithFlags(&P.ev_kb1[c], cudaEventDisableTiming));
    }
    CUDA_TRY(cudaEventCreateWithFlags(&P.ev_d2h, cudaEventDisableTiming));
    CUDA_TRY(cudaEventCreateWithFlags(&P.ev_start, cudaEventDisableTiming));
  }
  P.plan_for = h->var.func;
  return BLAST_CF_OK;
}

static int host_staging(blast_cf *h) {
  const size_t nx = (size_t)h->dim * h->nn, ne = (size_t)h->Z * h->nt, nr = (size_t)h->Z * h->nq;
  if (!h->d_in) {
    CUDA_TRY(cudaMalloc(&h->d_in, (2 * nx + ne + nr + 1) * sizeof(double)));
    CUDA_TRY(cudaMalloc(&h->d_out, (nx + ne + 1) * sizeof(double)));
  }
  return BLAST_CF_OK;
}

int blast_cf_set_rho0detJ0_host(blast_cf *h, const double *rho0detJ0) {
  if (!h || (!rho0detJ0 && h->Z > 0)) return fail(BLAST_CF_EINVAL, "NULL argument");
  int rc = check_async(h);
  if (rc || (rc = host_staging(h))) return rc;
  const size_t nx = (size_t)h->dim * h->nn, ne = (size_t)h->Z * h->nt, nr = (size_t)h->Z * h->nq;
  double *dr = h->d_in + 2 * nx + ne;
  if (nr) CUDA_TRY(cudaMemcpyAsync(dr, rho0detJ0, nr * sizeof(double), cudaMemcpyHostToDevice, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  h->rho_resident = true;
  return BLAST_CF_OK;
}

int blast_cf_eval_host(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                       double *out_Fdot1, double *out_FTv, double *out_dt_min) {
  NvtxRange nv("blast_cf_eval_host");
  if (!h) return fail(BLAST_CF_EINVAL, "handle is NULL");
  if (!out_dt_min || ((!x || !v || !out_Fdot1) && h->nn > 0) || ((!e || !out_FTv) && h->Z > 0))
    return fail(BLAST_CF_EINVAL, "NULL array argument");
  if (!rho0detJ0 && h->Z > 0 && !h->rho_resident)
    return fail(BLAST_CF_EINVAL, "rho0detJ0 is NULL and no resident copy was set (blast_cf_set_rho0detJ0_host)");
  int rc = check_async(h);
  if (rc) return rc;
  const size_t nx = (size_t)h->dim * h->nn, ne = (size_t)h->Z * h->nt, nr = (size_t)h->Z * h->nq;
  if ((rc = host_staging(h))) return rc;
  if (rho0detJ0) h->rho_resident = false;   // the upload below overwrites the resident copy
  if ((rc = host_plan(h))) return rc;
  blast_cf::HostPipe &P = h->hp;
  double *dx = h->d_in, *dv = dx + nx, *de = dv + nx, *dr = de + ne;
  double *dF = h->d_out, *dT = dF + nx, *dd = dT + ne;
  if (P.nch == 1 || h->timing || h->d_prof) {   // plain path: copy in, evaluate, copy out
    CUDA_TRY(cudaMemcpyAsync(dx, x, nx * sizeof(double), cudaMemcpyHostToDevice, h->stream));
    CUDA_TRY(cudaMemcpyAsync(dv, v, nx * sizeof(double), cudaMemcpyHostToDevice, h->stream));
    CUDA_TRY(cudaMemcpyAsync(de, e, ne * sizeof(double), cudaMemcpyHostToDevice, h->stream));
    if (rho0detJ0) CUDA_TRY(cudaMemcpyAsync(dr, rho0detJ0, nr * sizeof(double), cudaMemcpyHostToDevice, h->stream));
    if ((rc = blast_cf_eval(h, dx, dv, de, dr, dF, dT, dd))) return rc;
    CUDA_TRY(cudaMemcpyAsync(out_Fdot1, dF, nx * sizeof(double), cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaMemcpyAsync(out_FTv, dT, ne * sizeof(double), cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaMemcpyAsync(out_dt_min, dd, sizeof(double), cudaMemcpyDeviceToHost, h->stream));
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    return BLAST_CF_OK;
  }
  // the copy streams start after everything already queued on the handle's stream
  CUDA_TRY(cudaEventRecord(P.ev_start, h->stream));
  CUDA_TRY(cudaStreamWaitEvent(P.s_h2d, P.ev_start, 0));
  CUDA_TRY(cudaStreamWaitEvent(P.s_d2h, P.ev_start, 0));
  KB1Args a;
  a.zone_nodes = h->d_zone_nodes; a.J0inv = h->d_J0inv; a.J0inv_q = h->d_J0inv_q; a.zone_gamma = h->d_gamma; a.tab = h->d_tab;
  a.x = dx; a.v = dv; a.e = de; a.rho0detJ0 = dr; a.Fz1 = h->d_Fz1; a.FTv = dT; a.cta_dt = P.d_ctadt;
  a.Sq = nullptr; a.prof = nullptr; a.num_nodes = h->nn; a.zero = 0;
  a.ph.cfl = h->params.cfl; a.ph.q_quad = h->params.q_quad; a.ph.q_lin = h->params.q_lin;
  a.ph.eps_sw = h->params.eps_switch; a.ph.inv_2eps = 0.5 / h->params.eps_switch; a.ph.h0 = h->h0; a.ph.k = (double)h->k;
  a.ph.use_visc = h->params.use_viscosity; a.ph.use_vort = h->params.use_vorticity;
  int64_t done = 0;   // nodes [0, done) of x and v are on their way
  int64_t gathered = 0;   // nodes [0, gathered) of F.1 are gathered and on their way back
  for (int c = 0; c < P.nch; ++c) {
    const int64_t z0 = P.z0[c], zc = P.z0[c + 1] - z0, n1 = P.hi[c] + 1;
    if (n1 > done) {   // node range [done, n1) of every component: one 2D copy per array (rows of pitch nn)
      const size_t pitch = (size_t)h->nn * sizeof(double), w = (size_t)(n1 - done) * sizeof(double);
      CUDA_TRY(cudaMemcpy2DAsync(dx + done, pitch, x + done, pitch, w, h->dim, cudaMemcpyHostToDevice, P.s_h2d));
      CUDA_TRY(cudaMemcpy2DAsync(dv + done, pitch, v + done, pitch, w, h->dim, cudaMemcpyHostToDevice, P.s_h2d));
      done = n1;
    }
    CUDA_TRY(cudaMemcpyAsync(de + z0 * h->nt, e + z0 * h->nt, zc * h->nt * sizeof(double), cudaMemcpyHostToDevice, P.s_h2d));
    if (rho0detJ0)
      CUDA_TRY(cudaMemcpyAsync(dr + z0 * h->nq, rho0detJ0 + z0 * h->nq, zc * h->nq * sizeof(double),
                               cudaMemcpyHostToDevice, P.s_h2d));
    CUDA_TRY(cudaEventRecord(P.ev_in[c], P.s_h2d));
    CUDA_TRY(cudaStreamWaitEvent(h->stream, P.ev_in[c], 0));
    KB1Args ac = a;   // the same kernel on zones [z0, z0 + zc): zone-indexed arrays shifted
    ac.zone_nodes = h->d_zone_nodes + z0 * h->nk; ac.J0inv = h->d_J0inv + z0 * h->dim * h->dim;
    ac.zone_gamma = h->d_gamma + z0;
    if (h->d_J0inv_q) ac.J0inv_q = h->d_J0inv_q + z0 * h->nq * h->dim * h->dim;
    ac.e = de + z0 * h->nt; ac.rho0detJ0 = dr + z0 * h->nq; ac.Fz1 = h->d_Fz1 + z0 * h->dim * h->nk;
    ac.FTv = dT + z0 * h->nt; ac.cta_dt = P.d_ctadt + P.off[c]; ac.num_zones = zc;
    if (P.grid[c] > 0) h->var.launch(ac, P.grid[c], h->stream);
    CUDA_TRY(cudaEventRecord(P.ev_kb1[c], h->stream));
    CUDA_TRY(cudaStreamWaitEvent(P.s_d2h, P.ev_kb1[c], 0));
    CUDA_TRY(cudaMemcpyAsync(out_FTv + z0 * h->nt, dT + z0 * h->nt, zc * h->nt * sizeof(double), cudaMemcpyDeviceToHost,
                             P.s_d2h));
    // nodes below lo[c+1] touch no later chunk: gather them now and send their F.1 back while later chunks compute
    const int64_t g1 = c + 1 < P.nch ? P.lo[c + 1] : gathered;
    if (g1 > gathered) {
      launch_kb2(h, dF, nullptr, 0, nullptr, h->stream, gathered, g1);
      CUDA_TRY(cudaEventRecord(P.ev_kb1[c], h->stream));
      CUDA_TRY(cudaStreamWaitEvent(P.s_d2h, P.ev_kb1[c], 0));
      const size_t pitch = (size_t)h->nn * sizeof(double);
      CUDA_TRY(cudaMemcpy2DAsync(out_Fdot1 + gathered, pitch, dF + gathered, pitch, (g1 - gathered) * sizeof(double), h->dim,
                                 cudaMemcpyDeviceToHost, P.s_d2h));
      gathered = g1;
    }
  }
  // the remaining nodes and the min dt (nodes above hi[nch-1] belong to no zone: KB2 gives them F.1 = 0)
  launch_kb2(h, dF, P.d_ctadt, P.nslots, dd, h->stream, gathered, h->nn);
  if (h->nn > gathered) {
    const size_t pitch = (size_t)h->nn * sizeof(double);
    CUDA_TRY(cudaMemcpy2DAsync(out_Fdot1 + gathered, pitch, dF + gathered, pitch, (h->nn - gathered) * sizeof(double), h->dim,
                               cudaMemcpyDeviceToHost, h->stream));
  }
  CUDA_TRY(cudaMemcpyAsync(out_dt_min, dd, sizeof(double), cudaMemcpyDeviceToHost, h->stream));
  CUDA_TRY(cudaEventRecord(P.ev_d2h, P.s_d2h));
  CUDA_TRY(cudaStreamWaitEvent(h->stream, P.ev_d2h, 0));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  return check_async(h);
}

int blast_cf_eval_debug_Fz(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                           double *out_Fz) {
  if (!h || !out_Fz) return fail(BLAST_CF_EINVAL, "NULL argument");
  const size_t nx = (size_t)h->dim * h->nn, ne = (size_t)h->Z * h->nt;
  double *Sq = nullptr, *F1 = nullptr, *FT = nullptr;
  CUDA_TRY(cudaMalloc(&Sq, std::max<size_t>((size_t)h->Z * h->nq * h->dim * h->dim, 1) * sizeof(double)));
  CUDA_TRY(cudaMalloc(&F1, (nx + 1) * sizeof(double)));
  CUDA_TRY(cudaMalloc(&FT, (ne + 2) * sizeof(double)));
  int rc = eval_impl(h, x, v, e, rho0detJ0, F1, FT, FT + ne, Sq);
  if (!rc && h->Z > 0) {
    if (h->dim == 3) kbd_form_Fz<3><<<(int)h->Z, 128, 0, h->stream>>>(Sq, h->d_tab, h->k, h->Z, out_Fz);
    else kbd_form_Fz<2><<<(int)h->Z, 128, 0, h->stream>>>(Sq, h->d_tab, h->k, h->Z, out_Fz);
    if (cudaStreamSynchronize(h->stream) != cudaSuccess) rc = fail(BLAST_CF_ECUDA, "debug F_z kernel");
  }
  cudaFree(Sq); cudaFree(F1); cudaFree(FT);
  return rc;
}

int blast_cf_eval_loopback(blast_cf *const *hs, int n, const double *const *x, const double *const *v,
                           const double *const *e, const double *const *rho0detJ0, double *const *out_Fdot1,
                           double *const *out_FTv, double *const *out_dt_min) {
  if (!hs || n < 1 || !x || !v || !e || !rho0detJ0 || !out_Fdot1 || !out_FTv || !out_dt_min)
    return fail(BLAST_CF_EINVAL, "NULL argument");
  for (int r = 0; r < n; ++r) {
    if (!hs[r] || !hs[r]->xch || hs[r]->xch->comm || hs[r]->xch->nranks != n || hs[r]->xch->rank != r)
      return fail(BLAST_CF_EINVAL, "handle %d is not rank %d of a %d-rank loopback group", r, r, n);
  }
  int rc;
  bool all_overlap = true;
  for (int r = 0; r < n; ++r) all_overlap = all_overlap && hs[r]->xch->overlap;
  if (all_overlap) {
    // the overlap schedule of the NCCL path with device copies for the messages: per rank, KB1 on its
    // boundary zones, then (comm stream) the pack of its shared rows; the copies of a rank's recv rows wait
    // for its neighbours' packs; KB1 on the interior zones runs meanwhile on the rank's own stream
    std::vector<KB1Args> as(n);
    std::vector<int> gb(n), gi(n);
    for (int r = 0; r < n; ++r) {
      blast_cf *h = hs[r];
      if ((rc = check_async(h))) return rc;
      as[r] = make_args(h, x[r], v[r], e[r], rho0detJ0[r], out_FTv[r], nullptr);
      overlap_grids(h, h->xch->nb, h->Z - h->xch->nb, &gb[r], &gi[r]);
      if (h->timing) cudaEventRecord(h->ev[0], h->stream);
      CUDA_TRY(cudaEventRecord(h->xch->ev_s, h->stream));
      CUDA_TRY(cudaStreamWaitEvent(h->xch->s_comm, h->xch->ev_s, 0));
      launch_range(h, as[r], 0, h->xch->nb, gb[r], 0, h->xch->s_comm);   // boundary zones on the comm stream
      CUDA_TRY(cudaEventRecord(h->xch->ev_b, h->xch->s_comm));
      launch_pack_gather(h, h->xch->s_comm);
      CUDA_TRY(cudaEventRecord(h->xch->ev_p, h->xch->s_comm));
    }
    for (int r = 0; r < n; ++r) {   // "send / recv": rank r's recv rows from q are q's send rows for r
      blastcf::Exchange *xr = hs[r]->xch;
      for (int i = 0; i < xr->num_nbr; ++i) {
        const int q = xr->nbr_rank[i];
        blastcf::Exchange *xq = hs[q]->xch;
        int iq = -1;
        for (int t = 0; t < xq->num_nbr; ++t)
          if (xq->nbr_rank[t] == r) iq = t;
        const int64_t cnt = xr->nbr_offset[i + 1] - xr->nbr_offset[i];
        if (iq < 0 || xq->nbr_offset[iq + 1] - xq->nbr_offset[iq] != cnt)
          return fail(BLAST_CF_EINVAL, "ranks %d and %d disagree on their shared nodes", r, q);
        CUDA_TRY(cudaStreamWaitEvent(xr->s_comm, xq->ev_p, 0));
        CUDA_TRY(cudaMemcpyAsync(xr->d_recv + xr->nbr_offset[i] * xr->dim, xq->d_send + xq->nbr_offset[iq] * xq->dim,
                                 cnt * xr->dim * sizeof(double), cudaMemcpyDeviceToDevice, xr->s_comm));
      }
      if (hs[r]->timing) cudaEventRecord(xr->ev_sent, xr->s_comm);
    }
    for (int r = 0; r < n; ++r) {
      blast_cf *h = hs[r];
      blastcf::Exchange *xr = h->xch;
      launch_range(h, as[r], xr->nb, h->Z - xr->nb, gi[r], gb[r], h->stream);
      CUDA_TRY(cudaEventRecord(xr->ev_i, h->stream));
      if (h->timing) cudaEventRecord(h->ev[1], h->stream);
      CUDA_TRY(cudaStreamWaitEvent(xr->s_comm, xr->ev_i, 0));
      blastcf::xch_dt_reduce<<<1, 256, 0, xr->s_comm>>>(h->d_ctadt, gb[r] + gi[r], out_dt_min[r]);
      CUDA_TRY(cudaEventRecord(xr->ev_x, xr->s_comm));
      CUDA_TRY(cudaStreamWaitEvent(h->stream, xr->ev_b, 0));
      launch_kb2(h, out_Fdot1[r], nullptr, 0, xr->d_tmp, h->stream);
      if (h->timing) cudaEventRecord(h->ev[2], h->stream);
    }
    double dtg = HUGE_VAL, d;   // the allreduce(min): on the host in a loopback group
    for (int r = 0; r < n; ++r) {
      CUDA_TRY(cudaStreamSynchronize(hs[r]->xch->s_comm));
      CUDA_TRY(cudaMemcpyAsync(&d, out_dt_min[r], sizeof d, cudaMemcpyDeviceToHost, hs[r]->xch->s_comm));
      CUDA_TRY(cudaStreamSynchronize(hs[r]->xch->s_comm));
      dtg = std::min(dtg, d);
    }
    for (int r = 0; r < n; ++r) {
      blast_cf *h = hs[r];
      CUDA_TRY(cudaMemcpyAsync(out_dt_min[r], &dtg, sizeof dtg, cudaMemcpyHostToDevice, h->stream));
      CUDA_TRY(cudaStreamWaitEvent(h->stream, h->xch->ev_x, 0));
      blastcf::exchange_combine(h->xch, out_Fdot1[r]);
      if (h->timing) cudaEventRecord(h->ev[3], h->stream);
      CUDA_TRY(cudaStreamSynchronize(h->stream));
    }
    return check_async(hs[0]);
  }
  // 1. local corner force + gather on every partition, 2. pack shared-node partials
  for (int r = 0; r < n; ++r) {
    if ((rc = eval_impl(hs[r], x[r], v[r], e[r], rho0detJ0[r], out_Fdot1[r], out_FTv[r], out_dt_min[r], nullptr)))
      return rc;
    blastcf::exchange_pack(hs[r]->xch, out_Fdot1[r]);
  }
  for (int r = 0; r < n; ++r) CUDA_TRY(cudaStreamSynchronize(hs[r]->stream));
  // 3. the exchange: rank r's recv rows from q are rank q's send rows for r (same order: global node id)
  for (int r = 0; r < n; ++r) {
    blastcf::Exchange *xr = hs[r]->xch;
    for (int i = 0; i < xr->num_nbr; ++i) {
      const int q = xr->nbr_rank[i];
      blastcf::Exchange *xq = hs[q]->xch;
      int iq = -1;
      for (int t = 0; t < xq->num_nbr; ++t)
        if (xq->nbr_rank[t] == r) iq = t;
      const int64_t cnt = xr->nbr_offset[i + 1] - xr->nbr_offset[i];
      if (iq < 0 || xq->nbr_offset[iq + 1] - xq->nbr_offset[iq] != cnt)
        return fail(BLAST_CF_EINVAL, "ranks %d and %d disagree on their shared nodes", r, q);
      CUDA_TRY(cudaMemcpyAsync(xr->d_recv + xr->nbr_offset[i] * xr->dim, xq->d_send + xq->nbr_offset[iq] * xq->dim,
                               cnt * xr->dim * sizeof(double), cudaMemcpyDeviceToDevice, hs[r]->stream));
    }
  }
  // 4. global min dt
  double dtg = HUGE_VAL, d;
  for (int r = 0; r < n; ++r) {
    CUDA_TRY(cudaMemcpyAsync(&d, out_dt_min[r], sizeof d, cudaMemcpyDeviceToHost, hs[r]->stream));
    CUDA_TRY(cudaStreamSynchronize(hs[r]->stream));
    dtg = std::min(dtg, d);
  }
  // 5. ordered combine on every rank
  for (int r = 0; r < n; ++r) {
    CUDA_TRY(cudaMemcpyAsync(out_dt_min[r], &dtg, sizeof dtg, cudaMemcpyHostToDevice, hs[r]->stream));
    blastcf::exchange_combine(hs[r]->xch, out_Fdot1[r]);
    CUDA_TRY(cudaStreamSynchronize(hs[r]->stream));
  }
  return check_async(hs[0]);
}

int blast_cf_autotune(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                      double *out_Fdot1, double *out_FTv, double *out_dt_min, int reps, double *ms_out, int capacity,
                      int *num_candidates) {
  if (!h || !num_candidates) return fail(BLAST_CF_EINVAL, "NULL argument");
  const std::vector<KB1Variant> c = kb1_usable(h->dim, h->k, h->d_J0inv_q != nullptr);
  *num_candidates = (int)c.size();
  if (reps < 1) reps = 3;
  cudaEvent_t e0, e1;
  CUDA_TRY(cudaEventCreate(&e0));
  CUDA_TRY(cudaEventCreate(&e1));
  int best = 0;
  float best_ms = 1e30f;
  int rc = BLAST_CF_OK;
  for (size_t i = 0; i < c.size() && !rc; ++i) {
    if ((rc = apply_variant(h, c[i]))) break;
    if ((rc = blast_cf_eval(h, x, v, e, rho0detJ0, out_Fdot1, out_FTv, out_dt_min))) break;   // warm-up
    cudaEventRecord(e0, h->stream);
    for (int r = 0; r < reps && !rc; ++r) rc = blast_cf_eval(h, x, v, e, rho0detJ0, out_Fdot1, out_FTv, out_dt_min);
    cudaEventRecord(e1, h->stream);
    if (cudaEventSynchronize(e1) != cudaSuccess) { rc = fail(BLAST_CF_ECUDA, "autotune timing"); break; }
    float ms = 0.0f;
    cudaEventElapsedTime(&ms, e0, e1);
    ms /= reps;
    if (ms_out && (int)i < capacity) ms_out[i] = ms;
    if (ms < best_ms) { best_ms = ms; best = (int)i; }
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (rc) return rc;
  return c.empty() ? BLAST_CF_OK : apply_variant(h, c[best]);
}

const char *blast_cf_variant_name(const blast_cf *h, int index) {
  if (!h) return "";
  if (index < 0) return h->var.name ? h->var.name : "";
  static thread_local std::vector<KB1Variant> c;
  c = kb1_usable(h->dim, h->k, h->d_J0inv_q != nullptr);
  return index < (int)c.size() ? c[index].name : "";
}

int blast_cf_get_info(const blast_cf *h, blast_cf_info *info) {
  if (!h || !info) return fail(BLAST_CF_EINVAL, "NULL argument");
  info->dim = h->dim; info->order = h->k; info->nq = h->nq; info->nk = h->nk; info->nt = h->nt;
  info->num_zones = h->Z; info->num_nodes = h->nn; info->h0 = h->h0;
  info->zones_per_cta = h->var.zpc; info->threads_per_cta = h->var.nth; info->num_ctas = h->ncta;
  info->smem_bytes = h->var.smem; info->regs_per_thread = h->regs; info->local_bytes = h->local_bytes;
  info->flops_per_zone = flops_per_zone(h->dim, h->k);
  info->flops_per_zone_alg = flops_per_zone_alg(h->dim, h->k);
  // x, v read once, F.1 written once, e read, F^T v written, rho0|J0| read, dt
  info->alg_bytes = 8.0 * (3.0 * h->dim * h->nn + (double)h->Z * (2.0 * h->nt + h->nq)) + 8.0;
  info->kernels_per_eval = 2 + (h->xch ? blastcf::exchange_kernels(h->xch) : 0);
  return BLAST_CF_OK;
}

int blast_cf_set_timing(blast_cf *h, int enable) {
  if (!h) return fail(BLAST_CF_EINVAL, "handle is NULL");
  h->timing = enable != 0;
  return BLAST_CF_OK;
}

int blast_cf_debug_exchange_times(blast_cf *h, float *ms3) {
  if (!h || !ms3) return fail(BLAST_CF_EINVAL, "NULL argument");
  if (!h->timing || !h->xch || !h->xch->overlap) return fail(BLAST_CF_EINVAL, "timing off or no overlap schedule");
  CUDA_TRY(cudaEventSynchronize(h->ev[3]));
  CUDA_TRY(cudaEventElapsedTime(&ms3[0], h->ev[0], h->xch->ev_sent));
  CUDA_TRY(cudaEventElapsedTime(&ms3[1], h->ev[0], h->ev[1]));
  CUDA_TRY(cudaEventElapsedTime(&ms3[2], h->ev[0], h->ev[3]));
  return BLAST_CF_OK;
}

int blast_cf_exchange_schedule(const blast_cf *h, int32_t *mode, int64_t *boundary_zones) {
  if (!h || !mode) return fail(BLAST_CF_EINVAL, "NULL argument");
  *mode = h->xch ? (h->xch->overlap ? 2 : 1) : 0;
  if (boundary_zones) *boundary_zones = h->xch ? h->xch->nb : 0;
  return BLAST_CF_OK;
}

// ---- peer-memory transport (p2p.cuh) ----
namespace {
struct P2PRecord {   // + int64 recv_off[nranks], recv_cnt[nranks]
  char magic[8];
  cudaIpcMemHandle_t mem;
  uint64_t dptr;
  int32_t pid, device, rank, nranks, dim, overlap;
  int64_t nrows, mbox_bytes;
};
size_t p2p_record_bytes(int nranks) { return sizeof(P2PRecord) + 2 * sizeof(int64_t) * (size_t)nranks; }
struct DeviceGuard {   // the calling thread's current device, restored on return
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) == cudaSuccess && prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};
struct MboxLayout {   // byte offsets inside a mailbox (p2p.cuh)
  size_t rows, dt, flag_rows, flag_dt, ack, total;
};
MboxLayout mbox_layout(int64_t nrows, int dim, int nranks) {
  MboxLayout L;
  L.rows = 0;
  L.dt = L.rows + 2 * (size_t)std::max<int64_t>(nrows, 0) * dim * sizeof(double);
  L.flag_rows = L.dt + 2 * (size_t)nranks * sizeof(double);
  L.flag_dt = L.flag_rows + (size_t)nranks * sizeof(uint64_t);
  L.ack = L.flag_dt + (size_t)nranks * sizeof(uint64_t);
  L.total = L.ack + (size_t)nranks * sizeof(uint64_t);
  return L;
}
}  // namespace

int blast_cf_p2p_export(blast_cf *h, void *record, int64_t *bytes) {
  if (!h || !bytes) return fail(BLAST_CF_EINVAL, "NULL argument");
  if (!h->xch) return fail(BLAST_CF_EINVAL, "single-rank handle: nothing to exchange");
  blastcf::Exchange *x = h->xch;
  const size_t need = p2p_record_bytes(x->nranks);
  if (!record) {
    *bytes = (int64_t)need;
    return BLAST_CF_OK;
  }
  if (*bytes < (int64_t)need) return fail(BLAST_CF_EINVAL, "record buffer of %lld bytes, need %zu", (long long)*bytes, need);
  if (x->p2p.mapped) return fail(BLAST_CF_EINVAL, "already connected");
  DeviceGuard dg(h->device);
  const MboxLayout L = mbox_layout(x->nrows, x->dim, x->nranks);
  if (!x->p2p.mbox) {
    CUDA_TRY(cudaMalloc(&x->p2p.mbox, L.total));
    x->p2p.mbox_bytes = L.total;
  }
  // zero flags / acks before any peer can see the mailbox (its record leaves this process only after this)
  CUDA_TRY(cudaMemsetAsync(x->p2p.mbox, 0, L.total, h->stream));
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  std::vector<char> buf(need, 0);
  P2PRecord *r = reinterpret_cast<P2PRecord *>(buf.data());
  memcpy(r->magic, "BLASTP2P", 8);
  CUDA_TRY(cudaIpcGetMemHandle(&r->mem, x->p2p.mbox));
  r->dptr = (uint64_t)(uintptr_t)x->p2p.mbox;
  r->pid = (int32_t)getpid(); r->device = h->device; r->rank = x->rank; r->nranks = x->nranks; r->dim = x->dim;
  r->overlap = x->overlap ? 1 : 0; r->nrows = x->nrows; r->mbox_bytes = (int64_t)L.total;
  int64_t *off = reinterpret_cast<int64_t *>(r + 1), *cnt = off + x->nranks;
  for (int t = 0; t < x->nranks; ++t) { off[t] = -1; cnt[t] = 0; }
  for (int i = 0; i < x->num_nbr; ++i) {
    off[x->nbr_rank[i]] = x->nbr_offset[i];
    cnt[x->nbr_rank[i]] = x->nbr_offset[i + 1] - x->nbr_offset[i];
  }
  memcpy(record, buf.data(), need);
  *bytes = (int64_t)need;
  return BLAST_CF_OK;
}

int blast_cf_p2p_connect(blast_cf *h, const void *records, int64_t bytes_each) {
  if (!h || !records) return fail(BLAST_CF_EINVAL, "NULL argument");
  if (!h->xch) return fail(BLAST_CF_EINVAL, "single-rank handle: nothing to exchange");
  blastcf::Exchange *x = h->xch;
  blastcf::P2PHost &p = x->p2p;
  const int n = x->nranks, me = x->rank;
  if (bytes_each != (int64_t)p2p_record_bytes(n)) return fail(BLAST_CF_EINVAL, "record size %lld", (long long)bytes_each);
  if (!p.mbox || p.mapped || !p.peer.empty()) return fail(BLAST_CF_EINVAL, "export first, connect once");
  auto rec = [&](int t) { return reinterpret_cast<const P2PRecord *>(static_cast<const char *>(records) + (size_t)t * bytes_each); };
  auto roff = [&](int t) { return reinterpret_cast<const int64_t *>(rec(t) + 1); };
  for (int t = 0; t < n; ++t) {
    const P2PRecord *r = rec(t);
    if (memcmp(r->magic, "BLASTP2P", 8) != 0 || r->rank != t || r->nranks != n || r->dim != x->dim)
      return fail(BLAST_CF_EINVAL, "record %d is not rank %d of this %d-rank group", t, t, n);
  }
  if (rec(me)->dptr != (uint64_t)(uintptr_t)p.mbox || rec(me)->pid != (int32_t)getpid())
    return fail(BLAST_CF_EINVAL, "record %d is not this handle's", me);
  for (int i = 0; i < x->num_nbr; ++i) {   // both sides must agree on every shared row count
    const int q = x->nbr_rank[i];
    const int64_t mine = x->nbr_offset[i + 1] - x->nbr_offset[i];
    if (roff(q)[n + me] != mine || roff(q)[me] < 0)
      return fail(BLAST_CF_EINVAL, "ranks %d and %d disagree on their shared nodes", me, q);
  }
  DeviceGuard dg(h->device);
  p.peer.assign(n, nullptr);
  p.ipc_opened.assign(n, 0);
  for (int t = 0; t < n; ++t) {
    if (t == me) continue;
    const P2PRecord *r = rec(t);
    if (r->pid == (int32_t)getpid()) {   // same process: the allocation is addressable as is
      if (r->device != h->device) {
        int ok = 0;
        CUDA_TRY(cudaDeviceCanAccessPeer(&ok, h->device, r->device));
        if (!ok) return fail(BLAST_CF_EUNSUPPORTED, "device %d cannot access device %d", h->device, r->device);
        const cudaError_t e = cudaDeviceEnablePeerAccess(r->device, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) CUDA_TRY(e);
        cudaGetLastError();
      }
      p.peer[t] = (void *)(uintptr_t)r->dptr;
    } else {   // another process (device ordinals need not match across processes: the IPC open checks access)
      const cudaError_t e = cudaIpcOpenMemHandle(&p.peer[t], r->mem, cudaIpcMemLazyEnablePeerAccess);
      if (e != cudaSuccess) {
        p.peer[t] = nullptr;
        return fail(BLAST_CF_ECUDA, "cudaIpcOpenMemHandle(rank %d): %s", t, cudaGetErrorString(e));
      }
      p.ipc_opened[t] = 1;
    }
  }
  // device tables
  std::vector<double *> row_dst(std::max(x->num_nbr, 1), nullptr), dt_dst(n, nullptr);
  std::vector<int64_t> row_ps(std::max(x->num_nbr, 1), 0);
  std::vector<uint64_t *> row_flag(std::max(x->num_nbr, 1), nullptr), dt_flag(n, nullptr), ack_dst(n, nullptr);
  std::vector<int32_t> blk_off(x->num_nbr + 1, 0);
  for (int i = 0; i < x->num_nbr; ++i) {
    const int q = x->nbr_rank[i];
    const P2PRecord *r = rec(q);
    const MboxLayout Lq = mbox_layout(r->nrows, x->dim, n);
    row_dst[i] = reinterpret_cast<double *>(static_cast<char *>(p.peer[q]) + Lq.rows) + roff(q)[me] * x->dim;
    row_ps[i] = r->nrows * x->dim;
    row_flag[i] = reinterpret_cast<uint64_t *>(static_cast<char *>(p.peer[q]) + Lq.flag_rows) + me;
    const int64_t cnt = x->nbr_offset[i + 1] - x->nbr_offset[i];
    blk_off[i + 1] = blk_off[i] + (int32_t)std::min<int64_t>(std::max<int64_t>((cnt + 255) / 256, 1), 64);
  }
  for (int t = 0; t < n; ++t) {
    if (t == me) continue;
    const MboxLayout Lt = mbox_layout(rec(t)->nrows, x->dim, n);
    char *b = static_cast<char *>(p.peer[t]);
    dt_dst[t] = reinterpret_cast<double *>(b + Lt.dt);
    dt_flag[t] = reinterpret_cast<uint64_t *>(b + Lt.flag_dt) + me;
    ack_dst[t] = reinterpret_cast<uint64_t *>(b + Lt.ack) + me;
  }
  const size_t nn1 = std::max(x->num_nbr, 1);
  const size_t sz = nn1 * (sizeof(double *) + sizeof(int64_t) + sizeof(uint64_t *) + sizeof(int64_t) + sizeof(int32_t)) +
                    (size_t)n * (sizeof(double *) + 2 * sizeof(uint64_t *)) + (nn1 + 1) * sizeof(int32_t) +
                    (nn1 + 1) * sizeof(int32_t) + 64;
  CUDA_TRY(cudaMalloc(&p.d_tab, sz));
  CUDA_TRY(cudaMemset(p.d_tab, 0, sz));
  char *d = static_cast<char *>(p.d_tab);
  size_t o = 0;
  auto put = [&](const void *src, size_t bytes) -> void * {
    o = (o + 7) / 8 * 8;
    void *dst = d + o;
    if (bytes) cudaMemcpy(dst, src, bytes, cudaMemcpyHostToDevice);
    o += bytes;
    return dst;
  };
  std::vector<int64_t> nbr_off(x->nbr_offset.begin(), x->nbr_offset.end());
  if (nbr_off.empty()) nbr_off.push_back(0);
  std::vector<int32_t> nbr_rank(x->nbr_rank.begin(), x->nbr_rank.end());
  if (nbr_rank.empty()) nbr_rank.push_back(-1);
  blastcf::P2PDev &g = p.dev;
  g.row_dst = static_cast<double *const *>(put(row_dst.data(), nn1 * sizeof(double *)));
  g.row_pstride = static_cast<const int64_t *>(put(row_ps.data(), nn1 * sizeof(int64_t)));
  g.row_flag = static_cast<uint64_t *const *>(put(row_flag.data(), nn1 * sizeof(uint64_t *)));
  g.nbr_off = static_cast<const int64_t *>(put(nbr_off.data(), nbr_off.size() * sizeof(int64_t)));
  g.nbr_rank = static_cast<const int32_t *>(put(nbr_rank.data(), nbr_rank.size() * sizeof(int32_t)));
  g.blk_off = static_cast<const int32_t *>(put(blk_off.data(), blk_off.size() * sizeof(int32_t)));
  std::vector<int32_t> zeros(nn1 + 1, 0);
  g.cnt = static_cast<int32_t *>(put(zeros.data(), nn1 * sizeof(int32_t)));
  g.done = static_cast<int32_t *>(put(zeros.data(), sizeof(int32_t)));
  g.dt_dst = static_cast<double *const *>(put(dt_dst.data(), n * sizeof(double *)));
  g.dt_flag = static_cast<uint64_t *const *>(put(dt_flag.data(), n * sizeof(uint64_t *)));
  g.ack_dst = static_cast<uint64_t *const *>(put(ack_dst.data(), n * sizeof(uint64_t *)));
  if (o > sz) return fail(BLAST_CF_ECUDA, "p2p table overflow");
  CUDA_TRY(cudaGetLastError());
  g.num_nbr = x->num_nbr;
  const MboxLayout L = mbox_layout(x->nrows, x->dim, n);
  char *mb = static_cast<char *>(p.mbox);
  g.rows = reinterpret_cast<const double *>(mb + L.rows);
  g.rows_pstride = x->nrows * x->dim;
  g.dt = reinterpret_cast<const double *>(mb + L.dt);
  g.flag_rows = reinterpret_cast<const uint64_t *>(mb + L.flag_rows);
  g.flag_dt = reinterpret_cast<const uint64_t *>(mb + L.flag_dt);
  g.ack = reinterpret_cast<const uint64_t *>(mb + L.ack);
  g.me = me;
  g.nranks = n;
  p.send_blocks = blk_off[x->num_nbr];
  p.combine_blocks = (int)std::min<int64_t>(std::max<int64_t>((x->nu + 255) / 256, 1), 1184);
  // the schedule: overlap only if every rank can (the records carry each rank's own decision)
  bool all_overlap = true;
  for (int t = 0; t < n; ++t) all_overlap = all_overlap && rec(t)->overlap;
  x->overlap = all_overlap && x->overlap;
  p.epoch = 0;
  p.mapped = true;
  p.connected = true;
  CUDA_TRY(cudaDeviceSynchronize());
  return BLAST_CF_OK;
}

int blast_cf_p2p_enable(blast_cf *h, int enable) {
  if (!h || !h->xch) return fail(BLAST_CF_EINVAL, "not a multi-rank handle");
  blastcf::P2PHost &p = h->xch->p2p;
  if (enable && !p.mapped) return fail(BLAST_CF_EINVAL, "not connected");
  if (!enable && !h->xch->comm) return fail(BLAST_CF_EINVAL, "no NCCL communicator to fall back to");
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  p.connected = enable != 0;
  return BLAST_CF_OK;
}

int blast_cf_exchange_transport(const blast_cf *h, int32_t *transport) {
  if (!h || !transport) return fail(BLAST_CF_EINVAL, "NULL argument");
  *transport = !h->xch ? 0 : h->xch->p2p.connected ? 3 : h->xch->comm ? 1 : 2;
  return BLAST_CF_OK;
}

int blast_cf_kernel_times(blast_cf *h, float *ms3) {
  if (!h || !ms3) return fail(BLAST_CF_EINVAL, "NULL argument");
  if (!h->timing) return fail(BLAST_CF_EINVAL, "timing not enabled");
  CUDA_TRY(cudaEventSynchronize(h->ev[3]));
  CUDA_TRY(cudaEventElapsedTime(&ms3[0], h->ev[0], h->ev[1]));
  CUDA_TRY(cudaEventElapsedTime(&ms3[1], h->ev[1], h->ev[2]));
  CUDA_TRY(cudaEventElapsedTime(&ms3[2], h->ev[2], h->ev[3]));
  return BLAST_CF_OK;
}

int blast_cf_debug_cta_dt(blast_cf *h, double *host_out, int64_t capacity, int32_t *num_ctas, int32_t *zones_per_cta) {
  if (!h || !num_ctas || !zones_per_cta) return fail(BLAST_CF_EINVAL, "NULL argument");
  *num_ctas = h->ncta;
  *zones_per_cta = h->var.zpc;
  if (host_out && h->ncta > 0) {
    if (capacity < h->ncta) return fail(BLAST_CF_EINVAL, "capacity %lld < %d", (long long)capacity, h->ncta);
    CUDA_TRY(cudaStreamSynchronize(h->stream));
    CUDA_TRY(cudaMemcpy(host_out, h->d_ctadt, h->ncta * sizeof(double), cudaMemcpyDeviceToHost));
  }
  return BLAST_CF_OK;
}

int blast_cf_debug_stage_clocks(blast_cf *h, long long *host_out, int64_t capacity) {
  if (!h || !host_out) return fail(BLAST_CF_EINVAL, "NULL argument");
  if (!h->d_prof) return fail(BLAST_CF_EINVAL, "set BLAST_CF_PROFILE=1 before create");
  if (capacity < (int64_t)h->ncta * 16) return fail(BLAST_CF_EINVAL, "capacity");
  CUDA_TRY(cudaStreamSynchronize(h->stream));
  CUDA_TRY(cudaMemcpy(host_out, h->d_prof, (size_t)h->ncta * 16 * sizeof(long long), cudaMemcpyDeviceToHost));
  return BLAST_CF_OK;
}

int blast_cf_destroy(blast_cf *h) {
  if (!h) return fail(BLAST_CF_EINVAL, "handle is NULL");
  if (h->stream) cudaStreamSynchronize(h->stream);
  else cudaDeviceSynchronize();
  free_handle(h);
  return BLAST_CF_OK;
}

int blast_cf_exchange_plan(int32_t rank, int32_t num_neighbors, const int32_t *nbr_rank, const int64_t *nbr_offset,
                           const int32_t *nbr_nodes, int64_t capacity, int64_t *num_unique, int32_t *unique_nodes,
                           int64_t *src_ptr, int64_t *src) {
  if (num_neighbors < 0 || !num_unique || (num_neighbors > 0 && (!nbr_rank || !nbr_offset || !nbr_nodes)))
    return fail(BLAST_CF_EINVAL, "NULL argument");
  blastcf::ExchangePlan pl = blastcf::build_plan(rank, num_neighbors, nbr_rank, nbr_offset, nbr_nodes);
  *num_unique = (int64_t)pl.unique_nodes.size();
  if ((int64_t)pl.src.size() > capacity || (int64_t)pl.src_ptr.size() > capacity + 1)
    return fail(BLAST_CF_EINVAL, "capacity %lld too small", (long long)capacity);
  std::copy(pl.unique_nodes.begin(), pl.unique_nodes.end(), unique_nodes);
  std::copy(pl.src_ptr.begin(), pl.src_ptr.end(), src_ptr);
  std::copy(pl.src.begin(), pl.src.end(), src);
  return BLAST_CF_OK;
}

int blast_cf_owner_mask(int32_t rank, int32_t num_neighbors, const int32_t *nbr_rank, const int64_t *nbr_offset,
                        const int32_t *nbr_nodes, int64_t num_nodes, double *out) {
  if (num_neighbors < 0 || num_nodes < 0 || (num_nodes > 0 && !out) ||
      (num_neighbors > 0 && (!nbr_rank || !nbr_offset || !nbr_nodes)))
    return fail(BLAST_CF_EINVAL, "NULL argument");
  std::fill(out, out + num_nodes, 1.0);
  for (int i = 0; i < num_neighbors; ++i)   // the same rule as the integrator's owner weights
    if (nbr_rank[i] < rank)
      for (int64_t r = nbr_offset[i]; r < nbr_offset[i + 1]; ++r) {
        if (nbr_nodes[r] < 0 || nbr_nodes[r] >= num_nodes) return fail(BLAST_CF_EINVAL, "nbr_nodes[%lld]", (long long)r);
        out[nbr_nodes[r]] = 0.0;
      }
  return BLAST_CF_OK;
}

int blast_cf_nccl_unique_id_size(void) { return blastcf::nccl_unique_id_bytes(); }

int blast_cf_nccl_get_unique_id(void *out) {
  if (!out) return fail(BLAST_CF_EINVAL, "NULL argument");
  return blastcf::nccl_get_unique_id(out);
}

}  // extern "C"
