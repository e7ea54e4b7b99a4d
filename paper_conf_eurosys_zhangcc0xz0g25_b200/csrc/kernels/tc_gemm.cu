// tc_gemm.cu -- bf16 GEMM and implicit-GEMM convolution on the 5th-generation
// tensor cores (tcgen05.mma, fp32 accumulators in TMEM, operands staged by TMA),
// persistent under the SM-gated executor.
//
//   Y[M,N] = act((A[M,K] . B[N,K]^T) * scale[n] + shift[n] + R[M,N])   (bf16 out)
//
// A is X (GEMM) or the implicit im2col of an NHWC input (conv): an M tile is a
// BH x BW block of output pixels and, for every filter tap (r, s) and channel
// chunk, one TMA box load of the shifted input window -- out-of-bounds
// coordinates zero-fill, which implements the convolution padding.  Stride 2
// uses a rank-5 "parity" view of the input, (c, w%2, w/2, h%2, h/2), so every
// tap is again a dense box.  B is the KRSC weight matrix [Kout, R*S*C].
//
// Warp roles (320 threads): warp 0 = tile scheduler + TMA producer, warp 1 =
// MMA issuer (one thread) and TMEM owner, warps 2-5 = epilogue (TMEM -> regs ->
// fused epilogue -> global).  Tiles come from the executor's per-launch atomic
// queue; the TMEM accumulator is double buffered so the epilogue of tile i
// overlaps the main loop of tile i+1.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "../runtime/kdesc.hpp"
#include "executor.cuh"

namespace bless {

struct TcParams {
  CUtensorMap tmA;  // 64-byte aligned (first member of a 128-byte aligned block)
  CUtensorMap tmB;
  const float* scale;
  const float* shift;
  const __nv_bfloat16* R;
  __nv_bfloat16* Y;
  int M, N, K;
  int ldy, ldr, act;
  int mode;          // 0 GEMM, 1 conv stride 1 (4-D map), 2 conv stride 2 (5-D parity map)
  int tiles_n, num_kb;
  int OH, OW, BH, BW, tiles_w, C, R_, S_, pad, kc_per_tap;
  // split-K: work unit u -> (tile u / splits, K blocks [ks*kbs, min(num_kb, (ks+1)*kbs)))
  int splits, kbs;
  int stages;       // smem pipeline depth (runtime: budget / stage bytes, <= kMaxStages)
  float* ws;        // [tiles][128][BN] fp32 partial sums (zero between launches)
  unsigned* sem;    // [tiles] arrival counters (zero between launches)
  int sk_tiles;     // output tiles (workspace layout)
  // halo mode (3x3 stride-1 convs, HALO kernels): per 64-channel chunk ONE TMA
  // box of the tile's input halo ((BH+2) x BW pixels) serves all nine taps --
  // tap (r, s) is the same smem tile read from row r*BW + s on
  int astages;      // halo stages in smem (1 or 2)
  int a_stage_bytes;
  int a_tx;         // bytes one halo box delivers
  // weights in halo mode: one TMA box per filter row (the S taps of row r,
  // 3-D view (C, N, R*S) of the KRSC weights), so a 64-channel chunk costs
  // 1 + R boxes instead of 2 per tap (B200: a TMA box costs >= 130-180 ns per
  // SM whatever its size, profiles/round2/halo/tma_bench.txt)
  int b_stage_bytes;
  int taps_per_b;   // taps per weight box: S (one filter row, BN <= 64) or 1 (BN = 128: N >= 128 MMAs
                    // run at the tensor floor, N = 64 at ~60% of it; a 3-tap 128-wide box does not fit)
};

#ifdef __CUDACC__
// ------------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// Debug builds only (-DBLESS_TC_TRACE, tools/tctrace.py): per-CTA %globaltimer
// stamps of the pipeline phases of the last launch.
#ifdef BLESS_TC_TRACE
constexpr int kTrMax = 2048, kTrN = 13;
__device__ unsigned long long g_tc_trace[kTrMax][kTrN];
// latest CTA exit of any launch so far: read at griddepcontrol.wait's return
// (slot 12) it is the predecessor's last exit, so slot 4 - slot 12 = the
// programmatic-dependent-launch release latency
__device__ unsigned long long g_tc_last_exit;
__device__ __forceinline__ void tr_mark(int i) {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  if (blockIdx.x < kTrMax) g_tc_trace[blockIdx.x][i] = t;
  if (i == 9) atomicMax(&g_tc_last_exit, t);
  if (i == 4 && blockIdx.x < kTrMax) g_tc_trace[blockIdx.x][12] = *(volatile unsigned long long*)&g_tc_last_exit;
}
#define TR(i) tr_mark(i)
// wait accounting per CTA: [0] MMA warp waiting for operands (ns), [1] count,
// [2] producer waiting for free stages (ns), [3] count
__device__ unsigned long long g_tc_wait[kTrMax][4];
__device__ __forceinline__ unsigned long long tr_now() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define TW_BEGIN() const unsigned long long tw0_ = tr_now()
#define TW_END(slot) TW_END_K(slot, 0)
// + an event log of the first kEvCta CTAs: per role (0 MMA warp, 1 producer)
// {kind, time before the wait, time after it}; kind 1 weight/operand stage,
// 2 halo stage, 9 commit of a stage's MMAs (MMA warp)
constexpr int kEvCta = 8, kEvN = 192;
__device__ unsigned long long g_tc_ev[2][kEvCta][kEvN][3];
__device__ int g_tc_evn[2][kEvCta];
__device__ __forceinline__ void ev_log(int role, int& n, int kind, unsigned long long t0, unsigned long long t1) {
  if ((threadIdx.x & 31) == 0 && blockIdx.x < kEvCta && n < kEvN) {
    g_tc_ev[role][blockIdx.x][n][0] = kind;
    g_tc_ev[role][blockIdx.x][n][1] = t0;
    g_tc_ev[role][blockIdx.x][n][2] = t1;
    g_tc_evn[role][blockIdx.x] = ++n;
  }
}
#define TW_END_K(slot, kind) \
  { const unsigned long long tw1_ = tr_now(); \
    if ((threadIdx.x & 31) == 0 && blockIdx.x < kTrMax) { g_tc_wait[blockIdx.x][slot] += tw1_ - tw0_; g_tc_wait[blockIdx.x][slot + 1] += 1; } \
    ev_log(slot / 2, ev_n_, kind ? kind : 1, tw0_, tw1_); }
#define EV_COMMIT() { const unsigned long long tc_ = tr_now(); ev_log(0, ev_n_, 9, tc_, tc_); }
#define EV_DECL() int ev_n_ = 0
#else
#define TR(i) ((void)0)
#define TW_END_K(slot, kind) ((void)0)
#define EV_COMMIT() ((void)0)
#define EV_DECL() ((void)0)
#define TW_BEGIN() ((void)0)
#define TW_END(slot) ((void)0)
#endif

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// Warp-uniform wait (every lane polls, the loop exits on a warp vote): keeps
// the MMA warp's control flow provably convergent, so ptxas can keep the
// descriptor arithmetic on the uniform datapath instead of an ELECT +
// R2UR.BROADCAST sequence per tcgen05.mma.
__device__ __forceinline__ void mbar_wait_u(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  } while (!__all_sync(0xffffffffu, ok));
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
          smem_u32(dst)),
      "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(
          smem_u32(dst)),
      "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}
__device__ __forceinline__ void tma_load_4d(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1, int c2,
                                            int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], "
      "[%2];" ::"r"(smem_u32(dst)),
      "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
      : "memory");
}
__device__ __forceinline__ void tma_load_5d(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1, int c2,
                                            int c3, int c4) {
  asm volatile(
      "cp.async.bulk.tensor.5d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6, %7}], "
      "[%2];" ::"r"(smem_u32(dst)),
      "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4)
      : "memory");
}
// elected-lane TMA issue for the warp-uniform producer loop
#define BLESS_ELECT_ASM(body) "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t@e " body "\n\t}"
__device__ __forceinline__ void mbar_expect_tx_e(uint64_t* bar, uint32_t bytes) {
  asm volatile(BLESS_ELECT_ASM("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;") ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void tma_load_2d_e(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1) {
  asm volatile(BLESS_ELECT_ASM(
                   "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], "
                   "[%2];") ::"r"(smem_u32(dst)),
               "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void tma_load_3d_e(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1,
                                              int c2) {
  asm volatile(BLESS_ELECT_ASM("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, "
                               "{%3, %4, %5}], [%2];") ::"r"(smem_u32(dst)),
               "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2)
               : "memory");
}
__device__ __forceinline__ void tma_load_4d_e(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1, int c2,
                                              int c3) {
  asm volatile(BLESS_ELECT_ASM("cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, "
                               "{%3, %4, %5, %6}], [%2];") ::"r"(smem_u32(dst)),
               "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
               : "memory");
}
__device__ __forceinline__ void tma_load_5d_e(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1, int c2,
                                              int c3, int c4) {
  asm volatile(BLESS_ELECT_ASM("cp.async.bulk.tensor.5d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, "
                               "{%3, %4, %5, %6, %7}], [%2];") ::"r"(smem_u32(dst)),
               "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4)
               : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tc_mma(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc)
      : "memory");
}
// Warp-uniform issue: the whole MMA warp runs the loop, so descriptors and
// TMEM addresses live in uniform registers, and ONE elected lane issues.
// (Issuing from `if (lane == 0)` made ptxas wrap every tcgen05.mma in an
// ELECT + R2UR.BROADCAST waterfall loop: ~150 cycles per MMA instead of the
// 32-64 cycle tensor floor -- B200 phase traces, profiles/round2/mma_issue/.)
__device__ __forceinline__ void tc_mma_e(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                         uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p, e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc)
      : "memory");
}
__device__ __forceinline__ void tc_commit_e(uint64_t* bar) {
  asm volatile(
      "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_arrive_e(uint64_t* bar) {
  asm volatile(
      "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
      "@e mbarrier.arrive.shared::cta.b64 _, [%0];\n\t}" ::"r"(smem_u32(bar))
      : "memory");
}

// 32 lanes x 32 bit, 16 consecutive columns per thread
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),
        "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld_wait() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// UMMA shared-memory descriptor, K-major, swizzled (SW128/64/32: rows of
// BK*2 bytes, 8-row atoms; LBO = 16 B (unused for swizzled K-major), SBO =
// 8 rows * row bytes; version 1 = tcgen05; layout type 2/4/6).
// BK = 128 stages hold two 64-deep SW128 slabs (one TMA box each operand), so
// their descriptors are those of BK = 64.
template <int BK>
__device__ __forceinline__ uint64_t smem_desc(uint32_t saddr) {
  constexpr uint64_t row_bytes = (BK > 64 ? 64 : BK) * 2;
  constexpr uint64_t sbo = 8 * row_bytes;
  constexpr uint64_t layout = (BK >= 64) ? 2 : (BK == 32 ? 4 : 6);
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;                    // LBO (16 B)
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;  // SBO
  d |= (uint64_t)1 << 46;                    // version
  d |= layout << 61;
  return d;
}

// Same descriptor for a K-major SW128 tile that starts `row` 128-byte rows
// after a 1024-byte-aligned swizzle atom (the halo conv reads each tap's A
// tile at halo + (r*BW + s) rows).  Measured on B200 (profiles/round2/halo/):
// the hardware applies the 128-byte swizzle to the absolute shared-memory
// address bits, so a row-shifted start needs NO matrix base offset -- with
// base offset = (addr >> 7) & 7 the result is wrong, with 0 it is exact.
// -DBLESS_TC_HALO_BO=1 builds the other variant (probe only).
__device__ __forceinline__ uint64_t smem_desc_row(uint32_t saddr) {
#if defined(BLESS_TC_HALO_BO) && BLESS_TC_HALO_BO == 1
  return smem_desc<64>(saddr) | ((uint64_t)((saddr >> 7) & 7) << 49);
#else
  return smem_desc<64>(saddr);
#endif
}

// Instruction descriptor kind::f16: A, B bf16, D f32, both K-major, M = 128.
template <int BN>
__device__ __forceinline__ uint32_t instr_desc() {
  uint32_t d = 0;
  d |= 1u << 4;              // c_format = F32
  d |= 1u << 7;              // a_format = BF16
  d |= 1u << 10;             // b_format = BF16
  d |= (uint32_t)(BN >> 3) << 17;
  d |= (uint32_t)(128 >> 4) << 24;
  return d;
}

// Activation, resolved at compile time (the epilogue is instantiated per
// activation: a per-element switch serialised the 16-wide chunk).
// erf for the GELU epilogue: Abramowitz & Stegun 7.1.26 (|error| <= 1.5e-7,
// far below the bf16 output rounding of 2^-9), branch-free: one reciprocal,
// one exp2, nine FMAs -- erff's range split cost ~1 us per 128x64 tile
// (profiles/round1/tctrace_act.txt).
__device__ __forceinline__ float erf_as(float x) {
  const float ax = fabsf(x);
  const float t = __fdividef(1.f, fmaf(0.3275911f, ax, 1.f));
  float p = fmaf(1.061405429f, t, -1.453152027f);
  p = fmaf(p, t, 1.421413741f);
  p = fmaf(p, t, -0.284496736f);
  p = fmaf(p, t, 0.254829592f);
  const float e = 1.f - p * t * __expf(-ax * ax);
  return copysignf(e, x);
}

template <int ACT>
__device__ __forceinline__ float act_t(float y) {
  if (ACT == BL_ACT_RELU) return fmaxf(y, 0.f);
  if (ACT == BL_ACT_RELU6) return fminf(fmaxf(y, 0.f), 6.f);
  if (ACT == BL_ACT_GELU) return 0.5f * y * (1.f + erf_as(y * 0.70710678118654752f));
  return y;
}

// 256-bit global accesses (sm_100: LDG/STG.E.ENL2.256): one full 32-byte
// sector per lane -- half the store instructions of two 128-bit stores, and no
// half-sector writes, for the per-thread output rows of the epilogue.
__device__ __forceinline__ void st_global_256(void* ptr, const uint4& a, const uint4& b) {
  asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(ptr), "r"(a.x), "r"(a.y), "r"(a.z),
               "r"(a.w), "r"(b.x), "r"(b.y), "r"(b.z), "r"(b.w)
               : "memory");
}
__device__ __forceinline__ void ld_global_256(const void* ptr, uint4& a, uint4& b) {
  asm volatile("ld.global.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(a.x), "=r"(a.y), "=r"(a.z), "=r"(a.w), "=r"(b.x), "=r"(b.y), "=r"(b.z), "=r"(b.w)
               : "l"(ptr)
               : "memory");
}

// Fused epilogue for 16 consecutive columns of one output row:
// y = act(acc * scale + shift + R), rounded to bf16 (RNE), vector stores.
// sc/sh: the tile's per-column scale/shift staged in shared memory (1 / 0
// where absent), indexed from this 16-column chunk.
template <int ACT>
__device__ __forceinline__ void epi_store16(const TcParams& p, int m, int n0, float (&y)[16], const float* sc,
                                            const float* sh) {
  const bool full16 = n0 + 16 <= p.N;
#pragma unroll
  for (int i = 0; i < 16; ++i) y[i] = fmaf(y[i], sc[i], sh[i]);
  if (p.R) {
    const __nv_bfloat16* rr = p.R + (size_t)m * p.ldr + n0;
    if (full16 && ((p.ldr & 7) == 0)) {
      uint4 r0, r1;
      if ((((uintptr_t)rr) & 31) == 0) {
        ld_global_256(rr, r0, r1);
      } else {
        r0 = *reinterpret_cast<const uint4*>(rr);
        r1 = *reinterpret_cast<const uint4*>(rr + 8);
      }
      const __nv_bfloat16* e0 = reinterpret_cast<const __nv_bfloat16*>(&r0);
      const __nv_bfloat16* e1 = reinterpret_cast<const __nv_bfloat16*>(&r1);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        y[i] += __bfloat162float(e0[i]);
        y[8 + i] += __bfloat162float(e1[i]);
      }
    } else {
      for (int i = 0; i < 16; ++i)
        if (n0 + i < p.N) y[i] += __bfloat162float(rr[i]);
    }
  }
  __nv_bfloat16* yy = p.Y + (size_t)m * p.ldy + n0;
#ifdef BLESS_TC_NOSTORE   // debug experiment (tools/tctrace.py): epilogue without the global stores
  if (y[0] == 12345.f) *yy = __float2bfloat16_rn(y[1]);
  return;
#endif
  if (full16 && ((p.ldy & 7) == 0)) {
    uint4 o[2];
    __nv_bfloat162* ob = reinterpret_cast<__nv_bfloat162*>(o);
#pragma unroll
    for (int i = 0; i < 8; ++i) ob[i] = __floats2bfloat162_rn(act_t<ACT>(y[2 * i]), act_t<ACT>(y[2 * i + 1]));
    if ((((uintptr_t)yy) & 31) == 0) {
      st_global_256(yy, o[0], o[1]);
    } else {
      *reinterpret_cast<uint4*>(yy) = o[0];
      *reinterpret_cast<uint4*>(yy + 8) = o[1];
    }
  } else {
    for (int i = 0; i < 16; ++i)
      if (n0 + i < p.N) yy[i] = __float2bfloat16_rn(act_t<ACT>(y[i]));
  }
}

// Unsplit epilogue of one row (m) over this warp's columns [c0, c1) of the
// tile: TMEM -> registers (16 columns per wait) -> fused epilogue -> bf16.
// (Measured on B200, profiles/round1/tc_epilogue_ab.txt: the global stores
// cost ~2-3 us per 128x128 tile (-DBLESS_TC_NOSTORE: ffn1 12.8 -> 9.4 us), but
// warp-staging them through shared memory into full-sector row stores did not
// change the time, so the per-thread row stores stay.)
template <int ACT>
__device__ __forceinline__ void epi_cols(const TcParams& p, uint32_t tbase, int c0, int c1, int tn, int BN, int m,
                                         bool valid, const float* sc, const float* sh) {
#pragma unroll 1
  for (int c = c0; c < c1; c += 16) {
    uint32_t v[16];
    tmem_ld16(tbase + c, v);
    tmem_ld_wait();
    const int n0 = tn * BN + c;
    if (!valid || n0 >= p.N) continue;
    float y[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) y[i] = __uint_as_float(v[i]);
    epi_store16<ACT>(p, m, n0, y, sc + c, sh + c);
  }
}

// Split-K fp32 workspace layout: [tile][BN/16 column chunks][4 float4
// groups][128 rows][float4].  A thread owns one row (TMEM lane), so the four
// float4 of its 16-column chunk lie 2 KB apart and the 32 rows of a warp
// store/load 512 contiguous bytes per instruction (full sectors; the former
// row-major [row][BN] layout cost 32 partial-sector transactions per warp
// instruction and made the split-K epilogue ~4 us per 64 KB tile).
__device__ __forceinline__ float4* ws_at(const TcParams& p, int slab, int tile, int c, int i, int row, int BN) {
  const size_t chunk = ((size_t)slab * p.sk_tiles + tile) * (size_t)(BN >> 4) + (size_t)(c >> 4);
  return reinterpret_cast<float4*>(p.ws) + (chunk * 4 + i) * 128 + row;
}

template <int ACT>
__device__ __forceinline__ void epi_ws(const TcParams& p, int tile, int row, int c0, int c1, int tn, int BN, int m,
                                       const float* sc, const float* sh) {
#pragma unroll 1
  for (int c = c0; c < c1; c += 16) {
    const int n0 = tn * BN + c;
    if (n0 >= p.N) break;
    float y[16];
    float4 f[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) f[i] = __ldcg(ws_at(p, 0, tile, c, i, row, BN));
#pragma unroll
    for (int i = 0; i < 4; ++i) {   // re-zero for the next launch (after all four loads are issued)
      y[4 * i] = f[i].x; y[4 * i + 1] = f[i].y; y[4 * i + 2] = f[i].z; y[4 * i + 3] = f[i].w;
      __stcg(ws_at(p, 0, tile, c, i, row, BN), make_float4(0.f, 0.f, 0.f, 0.f));
    }
    epi_store16<ACT>(p, m, n0, y, sc + c, sh + c);
  }
}

#define TC_ACT_DISPATCH(act, CALL)                         \
  switch (act) {                                           \
    case BL_ACT_RELU: { constexpr int A_ = BL_ACT_RELU; CALL; } break;   \
    case BL_ACT_RELU6: { constexpr int A_ = BL_ACT_RELU6; CALL; } break; \
    case BL_ACT_GELU: { constexpr int A_ = BL_ACT_GELU; CALL; } break;   \
    default: { constexpr int A_ = BL_ACT_NONE; CALL; } break;           \
  }

constexpr int kEpiWarps = 8;   // 2 per SM sub-partition (TMEM lane quarter = warp % 4), split by columns
constexpr int kTcThreads = 64 + 32 * kEpiWarps;
constexpr int kMaxStages = 8;
constexpr int kDynSmemMax = 227 * 1024 - 2048;   // opt-in limit minus the executor's static smem

template <int BN, int BK, int MH = 1>
struct TcCfg {
  // MH = 2: the CTA's M tile is 256 rows -- one A box of 256 rows and TWO
  // M = 128 MMAs per K step sharing the B tile (twice the FLOPs per TMA box:
  // B200 charges a floor of ~130 ns per box)
  static constexpr int kStageA = MH * 128 * BK * 2;
  static constexpr int kStageB = BN * BK * 2;
  static constexpr int kStageBytes = kStageA + kStageB;
  // default pipeline: ~96 KB of stages, so two CTAs (the next kernel's, under
  // programmatic dependent launch, or another tenant's) fit on one SM
  static constexpr int kStages = std::max(2, std::min(6, (96 * 1024) / kStageBytes));
  // TMEM accumulators: double buffered (epilogue of tile i overlaps the MMAs of
  // tile i+1) up to BN = 128; BN = 256 keeps one so a second co-resident CTA
  // (another tenant's kernel on the same SM) can still allocate.
  static constexpr int kAcc = (BN * MH) >= 256 ? 1 : 2;
  static constexpr int kTmemCols = (kAcc * MH * BN) < 32 ? 32 : kAcc * MH * BN;
  static constexpr int kFixed = 1024 /*align*/ + 256 /*barriers*/ + 2 * BN * 4 /*sc, sh*/;
  static constexpr int kSmem = kStages * kStageBytes + kFixed;
  static constexpr int kSmemMax = kMaxStages * kStageBytes + kFixed;
};

template <int BN, int BK, bool HALO, int MH>
__device__ void tc_work(const TcParams& p, const GateArgs& g) {
  using Cfg = TcCfg<BN, BK, MH>;
  const int ST = p.stages;                           // B stages (A and B stages when !HALO)
  const int NA = HALO ? p.astages : ST;              // A stages
  const int a_bytes = HALO ? p.a_stage_bytes : Cfg::kStageA;
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  unsigned char* smem = (unsigned char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const int b_bytes = HALO ? p.b_stage_bytes : Cfg::kStageB;
  unsigned char* sA = smem;
  unsigned char* sB = smem + NA * a_bytes;
  unsigned char* bar_base = sB + ST * b_bytes;
  uint64_t* bars = (uint64_t*)bar_base;
  uint64_t* full = bars;            // [ST]
  uint64_t* empty = bars + ST;      // [ST]
  uint64_t* tfull = bars + 2 * ST;  // [2] accumulator ready
  uint64_t* tempty = tfull + 2;     // [2] accumulator drained
  uint64_t* rfull = tempty + 2;     // [2] tile ring
  uint64_t* rempty = rfull + 2;     // [2]
  uint64_t* fullA = rempty + 2;     // [2] halo stages (HALO)
  uint64_t* emptyA = fullA + 2;     // [2]
  int* ring = (int*)(emptyA + 2);   // [2]
  uint32_t* tmem_slot = (uint32_t*)(ring + 2);
  volatile int* last_flag = (volatile int*)(tmem_slot + 1);
  float* epi_sc = (float*)(bar_base + 256);  // [BN] tile scale
  float* epi_sh = epi_sc + BN;               // [BN] tile shift

  // warp index through a shuffle: provably warp-uniform, so role branches and
  // the MMA warp's loop stay on the uniform datapath
  const int warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0), lane = threadIdx.x & 31;
  EV_DECL();
  if (threadIdx.x == 0) TR(1);   // 1: work entry
  // the first tile claim (an L2 atomic round trip) overlaps the barrier/TMEM setup
  bool marked = false;
  int first_claim = -2;
  if (threadIdx.x == 0) first_claim = gate_claim(g, marked, false);
  if (threadIdx.x == 0) {
    for (int i = 0; i < ST; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&tfull[i], 1);
      mbar_init(&tempty[i], kEpiWarps);
      mbar_init(&rfull[i], 1);
      mbar_init(&rempty[i], 1 + kEpiWarps);
      mbar_init(&fullA[i], 1);
      mbar_init(&emptyA[i], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "n"(Cfg::kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  if (threadIdx.x == 0) TR(2);   // 2: barriers + TMEM ready
  // No grid-wide griddepcontrol.wait here: under programmatic dependent launch
  // the setup above, the first tile claim, the weight (B) loads and the
  // epilogue constants overlap the previous kernel; only reads of activations
  // (A operand, residual) and writes of the output wait for it.

  // debug experiments (tools/tctrace.py builds): drop one operand's loads or the MMAs
#ifdef BLESS_TC_SKIP_A
  constexpr bool kSkipA = true;
#else
  constexpr bool kSkipA = false;
#endif
#ifdef BLESS_TC_SKIP_B
  constexpr bool kSkipB = true;
#else
  constexpr bool kSkipB = false;
#endif
#ifdef BLESS_TC_SKIP_MMA
  constexpr bool kSkipMma = true;
#else
  constexpr bool kSkipMma = false;
#endif
  constexpr uint32_t kTxBytes = (kSkipA ? 0u : (uint32_t)Cfg::kStageA) + (kSkipB ? 0u : (uint32_t)Cfg::kStageB);
  if (warp == 0) {
    // ---------------- tile scheduler + TMA producer: the whole warp runs the
    // loop (uniform coordinates), lane 0 claims tiles, an elected lane issues
    if (lane == 0) {
      asm volatile("prefetch.tensormap [%0];" ::"l"(&p.tmA) : "memory");
      asm volatile("prefetch.tensormap [%0];" ::"l"(&p.tmB) : "memory");
    }
    {
      bool dep_waited = false;
      int stage = 0;
      uint32_t phase = 0;
      int astage = 0;
      uint32_t aphase = 0;
      int rs = 0;
      uint32_t rph = 0;
      for (;;) {
        int t0 = 0;
        if (lane == 0) t0 = first_claim != -2 ? first_claim : gate_claim(g, marked, dep_waited);
        const int t = __shfl_sync(0xffffffffu, t0, 0);
        first_claim = -2;
        if (!dep_waited && lane == 0) TR(3);          // 3: first claim returned
        mbar_wait(&rempty[rs], rph ^ 1);
        if (lane == 0) {
          ring[rs] = t;
          mbar_arrive(&rfull[rs]);
        }
        __syncwarp();
        if (++rs == 2) { rs = 0; rph ^= 1; }
        if (t < 0) {
          pdl_trigger();  // queue exhausted: let the next kernel on this stream launch
          break;
        }
        const int tile = t / p.splits, ks = t - tile * p.splits;
        const int kb0 = ks * p.kbs, kb1 = min(p.num_kb, kb0 + p.kbs);
        const int tm = tile / p.tiles_n, tn = tile - tm * p.tiles_n;
        int oh0 = 0, ow0 = 0;
        if (p.mode != 0) {
          const int th = tm / p.tiles_w;
          oh0 = th * p.BH;
          ow0 = (tm - th * p.tiles_w) * p.BW;
        }
        auto load_B = [&](int kb, int st) {
          unsigned char* b = sB + st * Cfg::kStageB;
          if (BK > 64) {   // 3-D view (64, N, K/64): one box = two 64-deep slabs
            const int kc = p.mode == 0 ? kb * 2 : (kb / p.kc_per_tap) * (p.C / 64) + (kb % p.kc_per_tap) * 2;
            tma_load_3d_e(b, &p.tmB, &full[st], 0, tn * BN, kc);
          } else if (p.mode == 0) {
            tma_load_2d_e(b, &p.tmB, &full[st], kb * BK, tn * BN);
          } else {
            const int tap = kb / p.kc_per_tap, c0 = (kb - tap * p.kc_per_tap) * BK;
            tma_load_2d_e(b, &p.tmB, &full[st], tap * p.C + c0, tn * BN);
          }
        };
        auto load_A = [&](int kb, int st) {
          unsigned char* a = sA + st * Cfg::kStageA;
          if (BK > 64 && p.mode == 0) {   // 3-D view (64, M, K/64)
            tma_load_3d_e(a, &p.tmA, &full[st], 0, tm * 128 * MH, kb * 2);
          } else if (BK > 64) {            // 4-D view (64, W, H, C/64), stride 1 only
            const int tap = kb / p.kc_per_tap, ch = (kb - tap * p.kc_per_tap) * 2;
            const int r = tap / p.S_, s = tap - r * p.S_;
            tma_load_4d_e(a, &p.tmA, &full[st], 0, ow0 - p.pad + s, oh0 - p.pad + r, ch);
          } else if (p.mode == 0) {
            tma_load_2d_e(a, &p.tmA, &full[st], kb * BK, tm * 128 * MH);
          } else {
            const int tap = kb / p.kc_per_tap, c0 = (kb - tap * p.kc_per_tap) * BK;
            const int r = tap / p.S_, s = tap - r * p.S_;
            if (p.mode == 1) {
              tma_load_4d_e(a, &p.tmA, &full[st], c0, ow0 - p.pad + s, oh0 - p.pad + r, 0);
            } else {
              const int dr = r - p.pad, ds = s - p.pad;
              const int ph = dr & 1, pw = ds & 1;        // parity of the input row/col
              const int qh = (dr - ph) / 2, qw = (ds - pw) / 2;
              tma_load_5d_e(a, &p.tmA, &full[st], c0, pw, ow0 + qw, ph, oh0 + qh);
            }
          }
        };
        if constexpr (HALO) {
          // per 64-channel chunk: the input halo once, then one weight box per filter row
          const int taps = p.R_ * p.S_ / p.taps_per_b;   // weight boxes per chunk
          auto load_Bt = [&](int c, int j) {
            { TW_BEGIN(); mbar_wait(&empty[stage], phase ^ 1); TW_END(2); }
            mbar_expect_tx_e(&full[stage], (uint32_t)b_bytes);
            tma_load_3d_e(sB + stage * b_bytes, &p.tmB, &full[stage], c * 64, tn * BN, j * p.taps_per_b);
            if (++stage == ST) { stage = 0; phase ^= 1; }
          };
          auto load_halo = [&](int c) {
            { TW_BEGIN(); mbar_wait(&emptyA[astage], aphase ^ 1); TW_END_K(2, 2); }
            mbar_expect_tx_e(&fullA[astage], (uint32_t)p.a_tx);
            tma_load_4d_e(sA + astage * a_bytes, &p.tmA, &fullA[astage], c * 64, -p.pad, oh0 - p.pad, 0);
            if (++astage == NA) { astage = 0; aphase ^= 1; }
          };
          for (int c = kb0; c < kb1; ++c) {
            int tap0 = 0;
            if (!dep_waited) {   // weights before the grid dependency resolves, activations after
              tap0 = min(taps, ST);
              for (int tap = 0; tap < tap0; ++tap) load_Bt(c, tap);
              dep_wait(g);
              if (t == 0 && lane == 0) gate_prev_end(g, (int64_t)ptx_globaltimer());
              if (lane == 0) TR(4);
              dep_waited = true;
            }
            load_halo(c);
            for (int tap = tap0; tap < taps; ++tap) load_Bt(c, tap);
          }
          continue;
        }
        int kb = kb0;
        if (!dep_waited) {
          // first tile: weights for up to ST stages before the grid dependency
          // resolves, activations after it
          const int npre = min(kb1 - kb0, ST);
          for (int i = 0; i < npre; ++i) {
            const int st = (stage + i) % ST;
            mbar_wait(&empty[st], (phase ^ (stage + i >= ST ? 1 : 0)) ^ 1);
            mbar_expect_tx_e(&full[st], kTxBytes);
            if (!kSkipB) load_B(kb0 + i, st);
          }
          dep_wait(g);
          if (t == 0 && lane == 0) gate_prev_end(g, (int64_t)ptx_globaltimer());   // predecessor just completed
          if (lane == 0) TR(4);          // 4: producer past griddepcontrol.wait
          dep_waited = true;
          for (int i = 0; i < npre; ++i)
            if (!kSkipA) load_A(kb0 + i, (stage + i) % ST);
          for (int i = 0; i < npre; ++i)
            if (++stage == ST) { stage = 0; phase ^= 1; }
          kb = kb0 + npre;
        }
        for (; kb < kb1; ++kb) {
          { TW_BEGIN(); mbar_wait(&empty[stage], phase ^ 1); TW_END(2); }
          mbar_expect_tx_e(&full[stage], kTxBytes);
          if (!kSkipB) load_B(kb, stage);
          if (!kSkipA) load_A(kb, stage);
          if (++stage == ST) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ---------------- MMA issuer (warp-uniform loop, elected issue)
    const uint32_t idesc = instr_desc<BN>();
    const uint32_t tmem_u = __shfl_sync(0xffffffffu, tmem_base, 0);
    int stage = 0;
    uint32_t phase = 0;
    int astage = 0;
    uint32_t aphase = 0;
    int rs = 0;
    uint32_t rph = 0;
    int acc = 0;
    uint32_t aph = 0;
    for (;;) {
      mbar_wait(&rfull[rs], rph);
      const int t = __shfl_sync(0xffffffffu, ring[rs], 0);
      __syncwarp();
      mbar_arrive_e(&rempty[rs]);
      if (++rs == 2) { rs = 0; rph ^= 1; }
      if (t < 0) break;
      const int ks = t % p.splits;
      const int kb0 = ks * p.kbs, kb1 = min(p.num_kb, kb0 + p.kbs);
      mbar_wait(&tempty[acc], aph ^ 1);
      tc_fence_after();
      const uint32_t d_tmem = tmem_u + acc * MH * BN;
      if constexpr (HALO) {
        for (int c = kb0; c < kb1; ++c) {
          { TW_BEGIN(); mbar_wait_u(&fullA[astage], aphase); TW_END_K(0, 2); }
          tc_fence_after();
          const uint32_t a_base = smem_u32(sA + astage * a_bytes);
          const int nbox = p.R_ * p.S_ / p.taps_per_b;
          int r = 0, s_ = 0;   // filter tap of the next MMA group (no division: uniform datapath)
          for (int j = 0; j < nbox; ++j) {   // one weight stage = taps_per_b consecutive taps
            { TW_BEGIN(); mbar_wait_u(&full[stage], phase); TW_END(0); }
            tc_fence_after();
            const uint32_t b_row = smem_u32(sB + stage * b_bytes);
            for (int u = 0; u < p.taps_per_b; ++u) {
              const uint32_t a0 = a_base + (uint32_t)(r * p.BW + s_) * 128u;
              const uint32_t b0 = b_row + (uint32_t)u * (BN * 128u);
              const uint32_t first = (c == kb0 && r == 0 && s_ == 0) ? 1u : 0u;
#pragma unroll
              for (int k = 0; k < 4; ++k)
                tc_mma_e(d_tmem, smem_desc_row(a0 + k * 32), smem_desc<64>(b0 + k * 32), idesc,
                         (first && k == 0) ? 0u : 1u);
              if (++s_ == p.S_) { s_ = 0; ++r; }
            }
            tc_commit_e(&empty[stage]);
            EV_COMMIT();
            __syncwarp();
            if (++stage == ST) { stage = 0; phase ^= 1; }
          }
          tc_commit_e(&emptyA[astage]);
          __syncwarp();
          if (++astage == NA) { astage = 0; aphase ^= 1; }
        }
      }
      for (int kb = HALO ? kb1 : kb0; kb < kb1; ++kb) {
        { TW_BEGIN(); mbar_wait_u(&full[stage], phase); TW_END(0); }
        tc_fence_after();
        if (lane == 0 && kb == kb0) TR(5);   // 5: first stage landed (last tile of this CTA)
        const uint32_t a0 = smem_u32(sA + stage * Cfg::kStageA);
        const uint32_t b0 = smem_u32(sB + stage * Cfg::kStageB);
        if (kSkipMma) {
          mbar_arrive_e(&empty[stage]);
        } else {
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            // BK = 128: slab k / 4 (128 x 64 of A, BN x 64 of B), K step k % 4
            const uint32_t ao = BK > 64 ? (k >> 2) * (128 * 128) + (k & 3) * 32 : k * 32;
            const uint32_t bo = BK > 64 ? (k >> 2) * (BN * 128) + (k & 3) * 32 : k * 32;
#pragma unroll
            for (int h = 0; h < MH; ++h)   // M half h: A rows 128h.. (SW128 rows of BK*2 bytes), accumulator h
              tc_mma_e(d_tmem + h * BN, smem_desc<BK>(a0 + h * (128 * BK * 2) + ao), smem_desc<BK>(b0 + bo), idesc,
                       (kb != kb0 || k) ? 1u : 0u);
          }
          tc_commit_e(&empty[stage]);
          EV_COMMIT();
        }
        __syncwarp();
        if (++stage == ST) { stage = 0; phase ^= 1; }
      }
      if (kSkipMma) mbar_arrive_e(&tfull[acc]);
      else tc_commit_e(&tfull[acc]);
      __syncwarp();
      if (++acc == Cfg::kAcc) { acc = 0; aph ^= 1; }
    }
  } else {
    // ---------------- epilogue warps 2..9: TMEM lane quarter = warp % 4, and
    // half (warp - 2) / 4 of the tile's columns, so every SM sub-partition
    // runs two epilogue warps
    const int q = warp & 3;
    const int half = (warp - 2) >> 2;
    const int c0 = BN >= 32 ? half * (BN / 2) : (half ? BN : 0);
    const int c1 = BN >= 32 ? c0 + BN / 2 : BN;
    bool dep_waited = false;
    int rs = 0;
    uint32_t rph = 0;
    int acc = 0;
    uint32_t aph = 0;
    for (;;) {
      mbar_wait(&rfull[rs], rph);
      const int t = ring[rs];
      __syncwarp();
      if (lane == 0) mbar_arrive(&rempty[rs]);
      if (++rs == 2) { rs = 0; rph ^= 1; }
      if (t < 0) break;
      const int tile = t / p.splits;
      const int tm = tile / p.tiles_n, tn = tile - tm * p.tiles_n;
      const int row = q * 32 + lane;
      // output row of this thread in M half h (MH = 2 only for GEMM / 1x1 tiles)
      auto out_row = [&](int h, int& m_, bool& valid_) {
        if (p.mode == 0) {
          m_ = (tm * MH + h) * 128 + row;
          valid_ = m_ < p.M;
        } else {
          const int th = tm / p.tiles_w;
          const int oh = th * p.BH + row / p.BW, ow = (tm - th * p.tiles_w) * p.BW + row % p.BW;
          valid_ = row < p.BH * p.BW && oh < p.OH && ow < p.OW;   // BH*BW < 128: tight halo tiles
          m_ = oh * p.OW + ow;
        }
      };
      int m;
      bool valid;
      out_row(0, m, valid);
      // stage this tile's scale/shift (independent of the previous kernel)
      asm volatile("bar.sync 2, %0;" ::"n"(32 * kEpiWarps) : "memory");   // previous tile's readers are done
      for (int i = threadIdx.x - 64; i < BN; i += 32 * kEpiWarps) {
        const int n = tn * BN + i;
        epi_sc[i] = (p.scale && n < p.N) ? __ldg(p.scale + n) : 1.f;
        epi_sh[i] = (p.shift && n < p.N) ? __ldg(p.shift + n) : 0.f;
      }
      asm volatile("bar.sync 2, %0;" ::"n"(32 * kEpiWarps) : "memory");
      if (!dep_waited) {   // residual reads / output writes depend on earlier kernels
        dep_wait(g);
        dep_waited = true;
      }
      for (int h = 0; h < MH; ++h) {   // pull this row's residual segment into L2 while the MMAs run
        int mh;
        bool vh;
        out_row(h, mh, vh);
        if (p.R && vh && c1 > c0) {
          const char* rr = reinterpret_cast<const char*>(p.R + (size_t)mh * p.ldr + tn * BN + c0);
          for (int b = 0; b < (c1 - c0) * 2; b += 128) asm volatile("prefetch.global.L2 [%0];" ::"l"(rr + b));
        }
      }
      mbar_wait(&tfull[acc], aph);
      tc_fence_after();
      if (threadIdx.x == 64) TR(6);      // 6: accumulator ready (last tile)
      const uint32_t tbase0 = tmem_base + ((uint32_t)(q * 32) << 16) + acc * MH * BN;
      if (p.splits == 1) {
        for (int h = 0; h < MH; ++h) {
          out_row(h, m, valid);
          const uint32_t tbase = tbase0 + h * BN;
          TC_ACT_DISPATCH(p.act, (epi_cols<A_>(p, tbase, c0, c1, tn, BN, m, valid, epi_sc, epi_sh)))
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[acc]);
        if (threadIdx.x == 64) TR(7);    // 7: epilogue stores issued (last tile)
        if (g.count_done) {   // software dependency: this unit's stores, then the count (release)
          asm volatile("bar.sync 1, %0;" ::"n"(32 * kEpiWarps) : "memory");
          if (threadIdx.x == 64)
            asm volatile("red.release.gpu.global.add.u64 [%0], 1;" ::"l"(&g.slot->done) : "memory");
        }
      } else {
        // split-K: add this unit's partial tile into the fp32 workspace
        // (sub-tile tile*MH + h per M half)
        for (int h = 0; h < MH; ++h) {
          out_row(h, m, valid);
          const uint32_t tbase = tbase0 + h * BN;
#pragma unroll 1
          for (int c = c0; c < c1; c += 16) {
            uint32_t v[16];
            tmem_ld16(tbase + c, v);
            tmem_ld_wait();
            if (!valid || tn * BN + c >= p.N) continue;
#pragma unroll
            for (int i = 0; i < 4; ++i)
              asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(
                               ws_at(p, 0, tile * MH + h, c, i, row, BN)),
                           "f"(__uint_as_float(v[4 * i])), "f"(__uint_as_float(v[4 * i + 1])),
                           "f"(__uint_as_float(v[4 * i + 2])), "f"(__uint_as_float(v[4 * i + 3]))
                           : "memory");
          }
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[acc]);  // TMEM no longer needed
        if (threadIdx.x == 64) TR(7);      // 7: partial-sum reds issued (split-K)
#ifdef BLESS_TC_SPLIT_FENCE_ALL   // A/B reference: every epilogue thread fences its own reds
        __threadfence();
#endif
        // release: the CTA barrier orders every epilogue thread's reds before
        // thread 64's gpu-scope release (cumulative), which is its arrival on
        // the tile's counter; one release per unit instead of 256
        asm volatile("bar.sync 1, %0;" ::"n"(32 * kEpiWarps) : "memory");   // all epilogue warps
        if (threadIdx.x == 64) {
#ifndef BLESS_TC_SPLIT_FENCE_ATOM
          // one acq_rel atomic: release of this unit's reds (ordered before it
          // by the barrier above), acquire of the other units' for the last one.
          // B200: 0.35-0.7 us less per split-K launch than fence + atomic +
          // fence (profiles/round2/splitk_acqrel/), same parity.
          unsigned prev_arr;
          asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(prev_arr) : "l"(p.sem + tile) : "memory");
          const bool last = prev_arr == (unsigned)p.splits - 1;
#else   // A/B reference: __threadfence + relaxed atomic (+ __threadfence on the last unit)
          __threadfence();
          const bool last = atomicAdd(p.sem + tile, 1u) == (unsigned)p.splits - 1;
          if (last) __threadfence();   // acquire: the other units' reds before our ld.cg reads
#endif
          *last_flag = last ? 1 : 0;
          TR(10);                          // 10: fence + tile counter arrival done (split-K)
        }
        asm volatile("bar.sync 1, %0;" ::"n"(32 * kEpiWarps) : "memory");
        if (*last_flag) {
#ifdef BLESS_TC_SPLIT_FENCE_ALL
          __threadfence();
#endif
          for (int h = 0; h < MH; ++h) {
            out_row(h, m, valid);
            if (valid) TC_ACT_DISPATCH(p.act, (epi_ws<A_>(p, tile * MH + h, row, c0, c1, tn, BN, m, epi_sc, epi_sh)))
          }
          if (threadIdx.x == 64) {
            p.sem[tile] = 0;
            TR(11);                        // 11: last unit's reduction epilogue done (split-K)
          }
        }
        if (g.count_done) {   // software dependency: partial (or the tile's final stores), then the count
          asm volatile("bar.sync 1, %0;" ::"n"(32 * kEpiWarps) : "memory");
          if (threadIdx.x == 64)
            asm volatile("red.release.gpu.global.add.u64 [%0], 1;" ::"l"(&g.slot->done) : "memory");
        }
      }
      if (++acc == Cfg::kAcc) { acc = 0; aph ^= 1; }
    }
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 1) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(Cfg::kTmemCols));
  }
  __syncthreads();
}

template <int BN, int BK, bool HALO, int MH>
__global__ void __launch_bounds__(kTcThreads, 2) k_tc_gemm(const __grid_constant__ TcParams p, const GateArgs g) {
  if (threadIdx.x == 0) TR(0);   // 0: CTA start
  // ONE inlined copy of tc_work (pass 0: in range / lingering; pass 1: the
  // exit protocol's fallback): with two copies ptxas moved the MMA warp's
  // descriptor arithmetic off the uniform datapath (an ELECT + 5 x
  // R2UR.BROADCAST sequence per tcgen05.mma, ~50 ns per MMA issued instead of
  // the tensor pipe's ~30)
  bool run = gate_in_range(g) || gate_linger(g);
  bool fb = false;
  int last = 0;
#pragma unroll 1
  for (int pass = 0; pass < 2; ++pass) {
    if (run) tc_work<BN, BK, HALO, MH>(p, g);
    if (pass == 1) break;
    pdl_trigger();
    if (threadIdx.x == 0) TR(8);   // 8: work done, before the exit atomic
    if (!g.stamp) {                // light exit
      if (threadIdx.x == 0) TR(9);
      return;
    }
    fb = gate_leave(g, last);
    run = fb;
    if (!fb) break;
  }
  if (last) gate_finalize(g, fb);
  if (threadIdx.x == 0) TR(9);   // 9: CTA exit
}
#endif  // __CUDACC__

// ------------------------------------------------------------------ host side
template <int BN, int BK, bool HALO, int MH>
static cudaError_t launch_tc(const KernelDesc& d, const GateArgs& g, cudaStream_t st) {
  void* args[2] = {(void*)d.params, (void*)&g};
  return launch_kernel((const void*)k_tc_gemm<BN, BK, HALO, MH>, dim3(launch_grid(d, g)), dim3(d.block),
                       (size_t)d.smem, st, args);
}

// Halo stages: NA halo stages + NB weight stages (one filter row each) within
// ~113 KB, so that two halo convs (or a halo conv and any other tile) still
// share an SM's 228 KB: two halo stages when two weight stages fit beside
// them (the next chunk's halo lands while this chunk's nine taps run), else
// one.  Returns false if not even 1 + 2 fit.  BLESS_TC_HALO_KB overrides the
// budget, BLESS_TC_HALO_NA=1 forces one halo stage (A/B sweeps).
static int halo_budget_kb() {
  const char* e = std::getenv("BLESS_TC_HALO_KB");
  return e ? std::max(64, std::min(226, std::atoi(e))) : 113;
}
template <int BN>
static bool halo_stages(const TcParams& p, int& na, int& nb) {
  using Cfg = TcCfg<BN, 64>;
  const int budget = halo_budget_kb() * 1024 - Cfg::kFixed;
  const char* fe = std::getenv("BLESS_TC_HALO_NA");
  const bool one = fe && std::atoi(fe) == 1;
  na = (!one && 2 * p.a_stage_bytes + 2 * p.b_stage_bytes <= budget) ? 2 : 1;
  nb = std::min(4, (budget - na * p.a_stage_bytes) / p.b_stage_bytes);
  return nb >= 2;
}

// Halo tile geometry: a tile is BH output rows of BW >= OW + 2 pixels (the
// halo row of every valid output column stays inside the tile row), BH*BW <=
// 128.  BW = OW + 2 exactly ("tight": 58 for OW = 56 -- a 30 KB halo stage, so
// two halo stages and two weight stages fit 113 KB) unless BLESS_TC_HALO_POW2=1
// (the power-of-two width of round 2's first halo kernel).  A stage holds the
// (BH + 2) x BW halo plus the rows the shifted tap views of the rows >= BH*BW
// (outputs discarded) can reach: row 127 + 2*BW + 2.
struct HaloGeo {
  int bw, bh, rows, a_stage;
};
static HaloGeo halo_geo(int OW) {
  const char* pe = std::getenv("BLESS_TC_HALO_POW2");
  const bool pow2 = pe && std::atoi(pe) != 0;
  HaloGeo g;
  g.bw = std::max(8, OW + 2);
  if (pow2) {
    int hw = 8;
    while (hw < OW + 2) hw <<= 1;
    g.bw = hw;
  }
  g.bh = 128 / g.bw;
  const int need = std::max((g.bh + 2) * g.bw, 130 + 2 * g.bw);
  g.rows = (need + 7) / 8 * 8;
  g.a_stage = (g.rows * 128 + 1023) / 1024 * 1024;
  return g;
}

template <int BN, int BK, bool HALO, int MH = 1>
static bool prep(KernelDesc& d, TcParams& p, std::string& err) {
  static std::once_flag once;
  static cudaError_t attr_err = cudaSuccess;
  std::call_once(once, [] {
    attr_err = cudaFuncSetAttribute((const void*)k_tc_gemm<BN, BK, HALO, MH>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    HALO ? kDynSmemMax : std::min(TcCfg<BN, BK, MH>::kSmemMax, kDynSmemMax));
  });
  if (attr_err != cudaSuccess) {
    err = std::string("cudaFuncSetAttribute: ") + cudaGetErrorString(attr_err);
    return false;
  }
  // pipeline depth: BLESS_TC_SMEM_KB overrides the ~96 KB default budget (sweeps)
  using Cfg = TcCfg<BN, BK, MH>;
  int st = Cfg::kStages;
  if (const char* e = std::getenv("BLESS_TC_SMEM_KB")) {
    const int kb = std::atoi(e);
    st = std::max(2, std::min(kMaxStages, (kb * 1024 - Cfg::kFixed) / Cfg::kStageBytes));
    while (st > 2 && st * Cfg::kStageBytes + Cfg::kFixed > kDynSmemMax) --st;
  }
  p.stages = st;
  d.smem = st * Cfg::kStageBytes + Cfg::kFixed;
  if (HALO) {
    int na = 1, nb = 2;
    if (!halo_stages<BN>(p, na, nb)) {
      err = "halo stages do not fit";
      return false;
    }
    p.astages = na;
    p.stages = nb;
    d.smem = na * p.a_stage_bytes + nb * p.b_stage_bytes + Cfg::kFixed;
  }
  d.launch = launch_tc<BN, BK, HALO, MH>;
  d.kernel_fn = (const void*)k_tc_gemm<BN, BK, HALO, MH>;
  d.counts_done = true;
  return true;
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn(std::string& err) {
  static EncodeTiledFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (EncodeTiledFn)f;
  });
  if (!fn) err = "cuTensorMapEncodeTiled unavailable";
  return fn;
}

static bool encode(CUtensorMap* map, int rank, const void* base, const cuuint64_t* dims, const cuuint64_t* strides,
                   const cuuint32_t* box, int BK, std::string& err) {
  EncodeTiledFn fn = encode_fn(err);
  if (!fn) return false;
  cuuint32_t es[5] = {1, 1, 1, 1, 1};
  const CUtensorMapSwizzle sw =
      BK >= 64 ? CU_TENSOR_MAP_SWIZZLE_128B : (BK == 32 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B);
  const CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, (cuuint32_t)rank, const_cast<void*>(base), dims,
                        strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    err = "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")";
    return false;
  }
  return true;
}

bool build_tc_gemm(const bl_op& op, const DeviceCaps& caps, KernelDesc& d, std::string& err, const TcChoice* force) {
  err.clear();
  if (op.dtype != BL_BF16 || caps.cc_major != 10) return false;
  TcParams p;
  std::memset(&p, 0, sizeof(p));
  p.scale = (const float*)op.ptr[2];
  p.shift = (const float*)op.ptr[3];
  p.R = (const __nv_bfloat16*)op.ptr[4];
  p.Y = (__nv_bfloat16*)op.ptr[5];
  p.act = op.act;
  const void* X = op.ptr[0];
  const void* W = op.ptr[1];
  int BK = 64;
  // BLESS_TC_CFG="BN,BK,splits" forces a tile configuration (sweeps only, tools/tcsweep.py)
  int fbn = 0, fbk = 0, fs = 0;
  if (const char* f = std::getenv("BLESS_TC_CFG")) std::sscanf(f, "%d,%d,%d", &fbn, &fbk, &fs);
  if (force && force->bk) fbk = force->bk;   // autotuner candidate (tc_candidates)
  const bool fbk_ok = fbk == 16 || fbk == 32 || fbk == 64 || fbk == 128;
  // BK = 128 stages (two 64-deep slabs per one 3-D/4-D TMA box): the K loop
  // pays a fixed cost per box, not per byte (profiles/round1/s4/tc_bk_sweep.txt),
  // so halving the boxes per K cuts 3x3 conv time 38-42% on B200
  // (s4/tc_bk128_ab.txt).  BLESS_TC_BK128=0 restores BK = 64 (A/B sweeps).
  static const bool bk128 = [] {
    const char* e = std::getenv("BLESS_TC_BK128");
    return !e || std::atoi(e) != 0;
  }();
  int lda = 0;   // A row pitch (elements) for a re-encode of the A map (MH = 2)
  if (op.kind == BL_OP_GEMM) {
    p.M = (int)op.dims[0];
    p.N = (int)op.dims[1];
    p.K = (int)op.dims[2];
    const int ldx = op.dims[3] ? (int)op.dims[3] : p.K;
    lda = ldx;
    p.ldy = op.dims[4] ? (int)op.dims[4] : p.N;
    p.ldr = op.dims[5] ? (int)op.dims[5] : p.N;
    if (p.M <= 8 || p.N % 16 || p.K % 8 || ldx % 8 || p.ldy % 8 || p.ldr % 8) return false;  // GEMV / SIMT
    if (((uintptr_t)X | (uintptr_t)W) & 15) return false;
    p.mode = 0;
    BK = fbk_ok ? fbk : ((bk128 && p.K % 64 == 0) ? 128 : 64);
    if (BK == 128 && p.K % 64) BK = 64;
    p.num_kb = (p.K + BK - 1) / BK;
    if (BK == 128) {   // (64, M, K/64): a box of two 64-deep slabs
      cuuint64_t da[3] = {64, (cuuint64_t)p.M, (cuuint64_t)(p.K / 64)}, sa[2] = {(cuuint64_t)ldx * 2, 128};
      cuuint32_t ba[3] = {64, 128, 2};
      if (!encode(&p.tmA, 3, X, da, sa, ba, BK, err)) return false;
    } else {
      cuuint64_t da[2] = {(cuuint64_t)p.K, (cuuint64_t)p.M}, sa[1] = {(cuuint64_t)ldx * 2};
      cuuint32_t ba[2] = {(cuuint32_t)BK, 128};
      if (!encode(&p.tmA, 2, X, da, sa, ba, BK, err)) return false;
    }
  } else if (op.kind == BL_OP_CONV) {
    const int Nb = (int)op.dims[0], H = (int)op.dims[1], Wd = (int)op.dims[2], C = (int)op.dims[3];
    const int K = (int)op.dims[4], R = (int)op.dims[5], S = (int)op.dims[6];
    const int stride = (int)op.dims[7], pad = (int)op.dims[8], groups = (int)op.dims[9];
    const int ldx = op.dims[10] ? (int)op.dims[10] : C;
    lda = ldx;
    p.ldy = op.dims[11] ? (int)op.dims[11] : K;
    p.ldr = p.ldy;
    const bool one_by_one = R == 1 && S == 1 && stride == 1 && pad == 0;
    if (Nb != 1 || groups != 1 || C % 8 || ldx % 8 || K % 8 || p.ldy % 8) return false;
    if (!one_by_one && C % 16) return false;
    if (stride != 1 && stride != 2) return false;
    if (stride == 2 && ((H | Wd) & 1)) return false;
    if (((uintptr_t)X | (uintptr_t)W) & 15) return false;
    // 1x1 stride-1 convs are plain GEMMs over pixels: any C % 8, K tail zero-filled by TMA
    BK = one_by_one ? 64 : ((C % 64 == 0) ? 64 : (C % 32 == 0 ? 32 : 16));
    if (bk128 && stride == 1 && (one_by_one ? C % 64 == 0 : C % 128 == 0)) BK = 128;
    if (fbk_ok && fbk < BK) BK = fbk;
    if (fbk == 128 && stride == 1 && (one_by_one ? C % 64 == 0 : C % 128 == 0)) BK = 128;
    p.OH = (H + 2 * pad - R) / stride + 1;
    p.OW = (Wd + 2 * pad - S) / stride + 1;
    p.M = p.OH * p.OW;
    p.N = K;
    p.K = R * S * C;
    p.C = C;
    p.R_ = R;
    p.S_ = S;
    p.pad = pad;
    p.kc_per_tap = one_by_one ? (C + BK - 1) / BK : C / BK;
    p.num_kb = R * S * p.kc_per_tap;
    // M tile = BH x BW output pixels (BH*BW = 128), BW the smallest power of two >= OW (<= 128)
    int BW = 1;
    while (BW < p.OW && BW < 128) BW <<= 1;
    BW = std::max(BW, 8);
    p.BW = BW;
    p.BH = 128 / BW;
    p.tiles_w = (p.OW + BW - 1) / BW;
    const int tiles_h = (p.OH + p.BH - 1) / p.BH;
    if (one_by_one && BK == 128) {
      p.mode = 0;
      cuuint64_t da[3] = {64, (cuuint64_t)(H * Wd), (cuuint64_t)(C / 64)}, sa[2] = {(cuuint64_t)ldx * 2, 128};
      cuuint32_t ba[3] = {64, 128, 2};
      if (!encode(&p.tmA, 3, X, da, sa, ba, BK, err)) return false;
    } else if (stride == 1 && BK == 128) {
      p.mode = 1;
      cuuint64_t da[4] = {64, (cuuint64_t)Wd, (cuuint64_t)H, (cuuint64_t)(C / 64)};
      cuuint64_t sa[3] = {(cuuint64_t)ldx * 2, (cuuint64_t)Wd * ldx * 2, 128};
      cuuint32_t ba[4] = {64, (cuuint32_t)BW, (cuuint32_t)p.BH, 2};
      if (!encode(&p.tmA, 4, X, da, sa, ba, BK, err)) return false;
    } else if (one_by_one) {
      // 1x1 stride-1: plain GEMM over pixels
      p.mode = 0;
      cuuint64_t da[2] = {(cuuint64_t)C, (cuuint64_t)(H * Wd)}, sa[1] = {(cuuint64_t)ldx * 2};
      cuuint32_t ba[2] = {(cuuint32_t)BK, 128};
      if (!encode(&p.tmA, 2, X, da, sa, ba, BK, err)) return false;
    } else if (stride == 1) {
      p.mode = 1;
      cuuint64_t da[4] = {(cuuint64_t)C, (cuuint64_t)Wd, (cuuint64_t)H, 1};
      cuuint64_t sa[3] = {(cuuint64_t)ldx * 2, (cuuint64_t)Wd * ldx * 2, (cuuint64_t)H * Wd * ldx * 2};
      cuuint32_t ba[4] = {(cuuint32_t)BK, (cuuint32_t)BW, (cuuint32_t)p.BH, 1};
      if (!encode(&p.tmA, 4, X, da, sa, ba, BK, err)) return false;
    } else {
      p.mode = 2;
      cuuint64_t da[5] = {(cuuint64_t)C, 2, (cuuint64_t)(Wd / 2), 2, (cuuint64_t)(H / 2)};
      cuuint64_t sa[4] = {(cuuint64_t)ldx * 2, (cuuint64_t)2 * ldx * 2, (cuuint64_t)Wd * ldx * 2,
                          (cuuint64_t)2 * Wd * ldx * 2};
      cuuint32_t ba[5] = {(cuuint32_t)BK, 1, (cuuint32_t)BW, 1, (cuuint32_t)p.BH};
      if (!encode(&p.tmA, 5, X, da, sa, ba, BK, err)) return false;
    }
    if (p.mode != 0) p.tiles_n = 0;  // set below
    (void)tiles_h;
    // halo mode: 3x3 "same" stride-1 conv, C % 64 == 0, and a tile row wide
    // enough that every valid output column's taps stay inside its halo row
    // (OW + 2 <= BW): one (64, BW, BH + 2) box per channel chunk serves all
    // nine taps (autotuner candidate, or BLESS_TC_HALO=1 as the default)
    const char* he = std::getenv("BLESS_TC_HALO");
    const int halo_env = he ? std::atoi(he) : 0;
    const bool want_halo = force ? force->halo != 0 : halo_env != 0;
    if (want_halo && stride == 1 && R == 3 && S == 3 && pad == 1 && C % 64 == 0 && p.OW + 2 <= 128) {
      const HaloGeo hg = halo_geo(p.OW);
      p.mode = 3;
      BK = 64;
      p.BW = hg.bw;
      p.BH = hg.bh;
      p.tiles_w = 1;
      p.kc_per_tap = C / 64;
      p.num_kb = C / 64;            // K blocks = channel chunks (nine taps each)
      p.a_stage_bytes = hg.a_stage;   // + the shifted-view overrun rows (only invalid outputs read them)
      p.a_tx = 64 * 2 * p.BW * (p.BH + 2);
      cuuint64_t da[4] = {(cuuint64_t)C, (cuuint64_t)Wd, (cuuint64_t)H, 1};
      cuuint64_t sa[3] = {(cuuint64_t)ldx * 2, (cuuint64_t)Wd * ldx * 2, (cuuint64_t)H * Wd * ldx * 2};
      cuuint32_t ba[4] = {64, (cuuint32_t)p.BW, (cuuint32_t)(p.BH + 2), 1};
      if (!encode(&p.tmA, 4, X, da, sa, ba, 64, err)) return false;
    }
  } else {
    return false;
  }
  // M tile of 256 rows (two M = 128 MMAs per K step sharing one B tile):
  // GEMM / 1x1 tiles with 64-deep stages (autotuner candidate, or BLESS_TC_MT=256)
  const char* mte = std::getenv("BLESS_TC_MT");
  const int want_mt = force ? force->mt : (mte ? std::atoi(mte) : 0);
  const int MH = (want_mt == 256 && p.mode == 0 && BK == 64) ? 2 : 1;
  if (MH == 2) {
    cuuint64_t da[2] = {(cuuint64_t)p.K, (cuuint64_t)p.M}, sa[1] = {(cuuint64_t)lda * 2};
    cuuint32_t ba[2] = {64, 256};
    if (!encode(&p.tmA, 2, X, da, sa, ba, 64, err)) return false;
  }
  // N tile: as wide as possible while keeping >= S tiles when the problem allows
  const int tiles_m = (p.mode == 0) ? (p.M + 128 * MH - 1) / (128 * MH) : p.tiles_w * ((p.OH + p.BH - 1) / p.BH);
  // N tile: the widest that still yields >= S tiles; if even 32 does not,
  // split K (>= 3 K blocks per work unit) until there are ~S work units, so a
  // batch-1 layer with few output tiles can still spread over every SM of its
  // range (SURVEY.md §8(d) "elastic" kernels).
  auto ntiles = [&](int bn) { return (long long)tiles_m * ((p.N + bn - 1) / bn); };
  int BN = p.N <= 16 ? 16 : (p.N <= 32 ? 32 : (p.N <= 64 ? 64 : 128));
  while (BN > 32 && ntiles(BN) < caps.S) BN >>= 1;
  p.tiles_n = (p.N + BN - 1) / BN;
  int splits = 1;
  if (ntiles(BN) < caps.S) {
    const int want = (int)((caps.S + ntiles(BN) - 1) / ntiles(BN));
    splits = std::max(1, std::min(want, p.mode == 3 ? p.num_kb : p.num_kb / 3));
  }
  if (force && force->bn) {
    fbn = force->bn;
    fs = force->splits;
  }
  if (fbn >= 16 && fbn <= 256 && (fbn & (fbn - 1)) == 0) {
    BN = fbn;
    p.tiles_n = (p.N + BN - 1) / BN;
  }
  if (BK == 128 && BN > 64) {
    // two BK = 128 stages must fit the ~96 KB budget that lets a second CTA
    // (another tenant's kernel under NSP) share the SM: BN <= 64.  BN = 128
    // stages of 64 KB cost co-residency and wrecked the C3/C4 squads on B200
    // (profiles/round1/s4/bench_bk128_bn128_*.json).
    BN = 64;
    p.tiles_n = (p.N + BN - 1) / BN;
  }
  if (MH == 2 && BN > 128) {   // 2 x 128 TMEM columns at most (one accumulator pair)
    BN = 128;
    p.tiles_n = (p.N + BN - 1) / BN;
  }
  if (p.mode == 3) {   // halo: the widest BN whose 1 halo + 2 weight stages fit (halo_stages)
    auto tpb = [&](int bn) { return bn >= 128 ? 1 : p.S_; };
    auto fits = [&](int bn) {
      const int fixed = 1024 + 256 + 2 * bn * 4;
      return p.a_stage_bytes + 2 * tpb(bn) * bn * 128 <= halo_budget_kb() * 1024 - fixed;
    };
    while (BN > 16 && !fits(BN)) BN >>= 1;
    p.tiles_n = (p.N + BN - 1) / BN;
    p.taps_per_b = tpb(BN);
  }
  if (fs >= 1) splits = std::min(fs, p.num_kb);
  p.kbs = (p.num_kb + splits - 1) / splits;
  p.splits = (p.num_kb + p.kbs - 1) / p.kbs;
  if (p.splits > 1) {
    const size_t nt = (size_t)ntiles(BN);
    // (a per-unit fp32 slab variant -- plain stores summed by the last unit --
    // was no faster on B200 and slower beyond 3 splits, profiles/round1/tc_splitk_*)
    p.sk_tiles = (int)nt * MH;   // workspace sub-tiles of 128 rows
    const size_t wsb = nt * MH * 128 * BN * sizeof(float);
    void* buf = nullptr;
    if (cudaMalloc(&buf, wsb + nt * sizeof(unsigned)) != cudaSuccess ||
        cudaMemset(buf, 0, wsb + nt * sizeof(unsigned)) != cudaSuccess) {
      err = "split-K workspace alloc";
      return false;
    }
    p.ws = (float*)buf;
    p.sem = (unsigned*)((char*)buf + wsb);
    d.owned = buf;
  }
  if (p.mode == 3) {
    p.b_stage_bytes = p.taps_per_b * BN * 128;
    cuuint64_t db[3] = {(cuuint64_t)p.C, (cuuint64_t)p.N, (cuuint64_t)(p.R_ * p.S_)};
    cuuint64_t sb[2] = {(cuuint64_t)p.K * 2, (cuuint64_t)p.C * 2};
    cuuint32_t bb[3] = {64, (cuuint32_t)BN, (cuuint32_t)p.taps_per_b};
    if (!encode(&p.tmB, 3, W, db, sb, bb, 64, err)) return false;
  } else if (BK == 128) {
    if (p.K % 64) { err = "BK 128 needs K % 64 == 0"; return false; }
    cuuint64_t db[3] = {64, (cuuint64_t)p.N, (cuuint64_t)(p.K / 64)}, sb[2] = {(cuuint64_t)p.K * 2, 128};
    cuuint32_t bb[3] = {64, (cuuint32_t)BN, 2};
    if (!encode(&p.tmB, 3, W, db, sb, bb, BK, err)) return false;
  } else {
    cuuint64_t db[2] = {(cuuint64_t)p.K, (cuuint64_t)p.N}, sb[1] = {(cuuint64_t)p.K * 2};
    cuuint32_t bb[2] = {(cuuint32_t)BK, (cuuint32_t)BN};
    if (!encode(&p.tmB, 2, W, db, sb, bb, BK, err)) return false;
  }
  d.op = op;
  d.tiles = (uint32_t)(tiles_m * p.tiles_n * p.splits);
  d.block = kTcThreads;
  d.grid = caps.S;
  // one CTA per SM on unrestricted launches (B200 kprobe: 0-4% faster than
  // two, profiles/round1/tc_occ.txt); restricted launches keep the
  // full-occupancy grid (launch_grid in kdesc.hpp)
  d.max_occ = 1;
  if (const char* e = std::getenv("BLESS_TC_MAX_OCC")) d.max_occ = std::max(1, std::atoi(e));   // sweeps
  bool ok = false;
#define TC_CASE(bn, bk) \
  if (BN == bn && BK == bk && p.mode != 3 && MH == 1) ok = prep<bn, bk, false>(d, p, err);
#define TC_MT2(bn) \
  if (BN == bn && BK == 64 && p.mode == 0 && MH == 2) ok = prep<bn, 64, false, 2>(d, p, err);
#define TC_HALO(bn) \
  if (BN == bn && p.mode == 3) ok = prep<bn, 64, true>(d, p, err);
  TC_CASE(16, 16) TC_CASE(16, 32) TC_CASE(16, 64)
  TC_CASE(32, 16) TC_CASE(32, 32) TC_CASE(32, 64)
  TC_CASE(64, 16) TC_CASE(64, 32) TC_CASE(64, 64)
  TC_CASE(128, 16) TC_CASE(128, 32) TC_CASE(128, 64)
  TC_CASE(256, 16) TC_CASE(256, 32) TC_CASE(256, 64)
  TC_CASE(16, 128) TC_CASE(32, 128) TC_CASE(64, 128)
  TC_HALO(16) TC_HALO(32) TC_HALO(64) TC_HALO(128)
  TC_MT2(32) TC_MT2(64) TC_MT2(128)
#undef TC_CASE
#undef TC_HALO
#undef TC_MT2
  if (!ok) {
    if (err.empty()) err = "no tc instantiation";
    return false;
  }
  static_assert(sizeof(TcParams) <= sizeof(d.params), "params block too small");
  std::memcpy(d.params, &p, sizeof(p));
  d.choice_bn = BN;
  d.choice_splits = p.splits;
  d.choice_bk = BK;
  d.choice_halo = p.mode == 3 ? 1 : 0;
  d.choice_mt = 128 * MH;
  d.family = op.kind == BL_OP_GEMM ? "tc_gemm_bf16" : (p.mode == 0 ? "tc_conv1x1_bf16" : "tc_conv_bf16");
  if (BK == 128 && BN > 64 && p.mode == 3) { err = "halo BN"; return false; }
  d.flops = 2.0 * p.M * p.N * p.K;
  double a_bytes = (op.kind == BL_OP_CONV) ? 2.0 * op.dims[1] * op.dims[2] * op.dims[3] : 2.0 * p.M * p.K;
  d.bytes = a_bytes + 2.0 * p.N * p.K + 2.0 * p.M * p.N * (p.R ? 2 : 1);
  return true;
}

// Candidate tile configurations for the registration-time autotuner
// (DeviceRT::add_kernel): BN in {32, 64, 128} (narrower when N is small) x BK
// in {64, 128} (128 only where build_tc_gemm takes it -- K % 64 == 0 for GEMMs
// and 1x1 convs, C % 128 == 0 for stride-1 3x3 convs -- and only with
// BN <= 64, which keeps two stages in the ~96 KB co-residency budget), each
// unsplit and split-K to about S work units.  Measured on B200
// (tools/tcsweep.py, profiles/round1/tcsweep.txt, s4/tc_bk128_ab.txt) no single
// rule picks the fastest: unsplit tiles below S often win (split-K's fp32
// reduction costs several us), BK = 128 wins the 3x3 convs, BN = 128 with
// BK = 64 wins large GEMMs; BN = 256 never won with 96 KB of stages.
int tc_candidates(const bl_op& op, const DeviceCaps& caps, TcChoice* out, int max) {
  long long M = 0, N, num_kb, tiles_m, halo_tiles_m = 0, chunks = 0, halo_a_stage = 0;
  bool bk128_ok = false, halo_ok = false, gemm_like = false;
  if (op.kind == BL_OP_GEMM) {
    M = op.dims[0], N = op.dims[1];
    num_kb = (op.dims[2] + 63) / 64;
    tiles_m = (M + 127) / 128;
    bk128_ok = op.dims[2] % 64 == 0;
    gemm_like = true;
  } else if (op.kind == BL_OP_CONV) {
    const long long H = op.dims[1], W = op.dims[2], C = op.dims[3], R = op.dims[5], S = op.dims[6];
    const long long st = op.dims[7] ? op.dims[7] : 1, pad = op.dims[8];
    const long long OH = (H + 2 * pad - R) / st + 1, OW = (W + 2 * pad - S) / st + 1;
    const bool one = R == 1 && S == 1 && st == 1 && pad == 0;
    N = op.dims[4];
    num_kb = R * S * std::max(1LL, C / 64);
    long long BW = 8;
    while (BW < OW && BW < 128) BW <<= 1;
    tiles_m = ((OW + BW - 1) / BW) * ((OH + (128 / BW) - 1) / (128 / BW));
    bk128_ok = st == 1 && (one ? C % 64 == 0 : C % 128 == 0);
    gemm_like = one;
    M = OH * OW;
    halo_ok = st == 1 && R == 3 && S == 3 && pad == 1 && C % 64 == 0 && OW + 2 <= 128;
    if (halo_ok) {
      const HaloGeo hg = halo_geo((int)OW);
      halo_tiles_m = (OH + hg.bh - 1) / hg.bh;
      halo_a_stage = hg.a_stage;
    }
    chunks = C / 64;
  } else {
    return 0;
  }
  int n = 0;
  const int nmax = N <= 16 ? 16 : (N <= 32 ? 32 : (N <= 64 ? 64 : 128));
  const char* he = std::getenv("BLESS_TC_HALO");   // "0": no halo candidates (A/B sweeps)
  if (halo_ok && !(he && std::atoi(he) == 0)) {
    // halo tiles: BH x BW with BW >= OW + 2; K blocks = 64-channel chunks
    for (int bn = std::min(32, nmax); bn <= nmax && n < max; bn <<= 1) {
      const int tpb = bn >= 128 ? 1 : 3;
      if (halo_a_stage + 2 * tpb * bn * 128 > halo_budget_kb() * 1024 - (1024 + 256 + 2 * bn * 4)) break;
      const long long tiles = halo_tiles_m * ((N + bn - 1) / bn);
      out[n++] = TcChoice{bn, 1, 64, 1};
      if (tiles < caps.S && chunks >= 2 && n < max) {
        const long long want = std::min<long long>((caps.S + tiles - 1) / tiles, chunks);
        if (want >= 2) out[n++] = TcChoice{bn, (int)want, 64, 1};
      }
    }
  }
  if (gemm_like && M >= 1024) {
    // M tiles of 256 rows (two M = 128 MMAs per K step): half the tiles, twice
    // the FLOPs per TMA box; only where M leaves enough tiles (B200: never
    // faster on the configs' batch-1 GEMMs at ~96 KB of stages, 1.33x on a
    // large HBM-streaming GEMM with 160-200 KB, profiles/round2/mt256/)
    const long long tiles_m2 = (M + 255) / 256;
    for (int bn = std::min(64, nmax); bn <= nmax && n < max; bn <<= 1) {
      const long long tiles = tiles_m2 * ((N + bn - 1) / bn);
      out[n++] = TcChoice{bn, 1, 64, 0, 256};
      if (tiles < caps.S && num_kb >= 6 && n < max) {
        const long long want = std::min<long long>((caps.S + tiles - 1) / tiles, num_kb / 3);
        if (want >= 2) out[n++] = TcChoice{bn, (int)want, 64, 0, 256};
      }
    }
  }
  for (int bn = std::min(32, nmax); bn <= nmax; bn <<= 1) {
    for (int bk = 64; bk <= 128; bk += 64) {
      if (bk == 128 && (!bk128_ok || bn > 64)) continue;
      const long long kbs = bk == 128 ? (num_kb + 1) / 2 : num_kb;   // K blocks at this depth
      const long long tiles = tiles_m * ((N + bn - 1) / bn);
      if (n < max) out[n++] = TcChoice{bn, 1, bk};
      if (tiles < caps.S && kbs >= 6) {
        const long long want = std::min<long long>((caps.S + tiles - 1) / tiles, kbs / 3);
        if (want >= 2 && n < max) out[n++] = TcChoice{bn, (int)want, bk};
        if (want >= 6 && n < max) out[n++] = TcChoice{bn, (int)(want / 2), bk};
      }
    }
  }
  return n;
}

}  // namespace bless

#ifdef BLESS_TC_TRACE
// debug builds only: copy the per-CTA phase stamps out (tools/tctrace.py)
extern "C" int bl_debug_tc_trace(unsigned long long* host, int n_cta) {
  const size_t n = (size_t)std::min(n_cta, bless::kTrMax) * bless::kTrN * sizeof(unsigned long long);
  return (int)cudaMemcpyFromSymbol(host, bless::g_tc_trace, n);
}
extern "C" int bl_debug_tc_wait(unsigned long long* host, int n_cta) {
  const size_t n = (size_t)std::min(n_cta, bless::kTrMax) * 4 * sizeof(unsigned long long);
  return (int)cudaMemcpyFromSymbol(host, bless::g_tc_wait, n);
}
extern "C" int bl_debug_tc_events(unsigned long long* host, int* counts) {
  cudaMemcpyFromSymbol(counts, bless::g_tc_evn, sizeof(bless::g_tc_evn));
  return (int)cudaMemcpyFromSymbol(host, bless::g_tc_ev, sizeof(bless::g_tc_ev));
}
extern "C" int bl_debug_tc_trace_clear() {
  static int zn[2][bless::kEvCta];
  cudaMemcpyToSymbol(bless::g_tc_evn, zn, sizeof(zn));
  static unsigned long long z[bless::kTrMax][bless::kTrN];
  static unsigned long long zw[bless::kTrMax][4];
  cudaMemcpyToSymbol(bless::g_tc_wait, zw, sizeof(zw));
  return (int)cudaMemcpyToSymbol(bless::g_tc_trace, z, sizeof(z));
}
#endif
