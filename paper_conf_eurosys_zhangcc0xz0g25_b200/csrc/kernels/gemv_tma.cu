// gemv_tma.cu -- batch-1 fully-connected layers (M <= 8 rows of X) as an HBM
// weight stream, under the SM-gated executor (SURVEY.md K2 GEMV shapes: VGG
// FC 25088->4096->4096->1000, ResNet FC 2048->1000).
//
//   Y[m, n] = act((sum_k X[m, k] W[n, k]) * scale[n] + shift[n] + R[m, n])
//
// A work tile is a block of `rows` (1, 2, 4 or 8) consecutive rows of W, i.e.
// one contiguous rows*K*2-byte region.  Warp 0 (one thread) streams it into a
// ring of 16 KB shared-memory stages with cp.async.bulk (TMA bulk copies,
// completion via mbarrier transaction counts) and keeps streaming into the
// next claimed tile, so an SM always has kStages*16 KB of weights in flight.
// A stage holds rows x (8192/rows) k-values, so it is full whatever the tile
// height: 16/rows consumer warps share a row, each owning a 512-k window of
// every stage (16 consecutive k per lane), and keep one running dot product
// per X row that is folded into shared-memory row partials once per tile.
// Short tiles (rows < 8) keep the dynamic queue's tail short: the last tile an
// SM pulls is rows*K*2 bytes, ~9 us of one SM's HBM share at rows = 8 for VGG
// FC1.  HBM-bound: no tensor cores (the contraction has M <= 8).
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdlib>
#include <cstring>
#include <mutex>

#include "../runtime/kdesc.hpp"
#include "executor.cuh"

namespace bless {

struct GemvTmaParams {
  const __nv_bfloat16* X;
  const __nv_bfloat16* W;
  const float* scale;
  const float* shift;
  const __nv_bfloat16* R;
  __nv_bfloat16* Y;
  int M, N, K, ldx, ldy, ldr, act;
  int rows;       // rows of W per tile
  float invK;     // 1 / K (row index of a run by reciprocal multiply)
  int warp_rows;  // K % 512 == 0: a warp's 512-element window never straddles two rows
};

constexpr int kGvStage = 16384;               // bytes per stage
#ifndef BLESS_GEMV_STAGES
#define BLESS_GEMV_STAGES 6
#endif
constexpr int kGvStages = BLESS_GEMV_STAGES;
constexpr int kGvElems = kGvStage / 2;        // bf16 elements per stage
constexpr int kGvConsumers = 16;              // consumer warps
constexpr int kGvRun = 16;                    // k values per lane per stage
constexpr int kGvWin = 32 * kGvRun;            // k values per consumer warp per stage (512)
constexpr int kGvThreads = 32 * (1 + kGvConsumers);
constexpr int kGvMaxRows = 8;
constexpr int kGvSmem = kGvStages * kGvStage + 1024 + 8 * kGvMaxRows * 4 + 256;
static_assert(kGvRun == 16, "run length");

#ifdef __CUDACC__
__device__ __forceinline__ uint32_t gv_smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void gv_mbar_init(uint64_t* b, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(gv_smem_u32(b)), "r"(c));
}
__device__ __forceinline__ void gv_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(gv_smem_u32(b)) : "memory");
}
__device__ __forceinline__ void gv_expect(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(gv_smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void gv_wait(uint64_t* b, uint32_t par) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tW_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra W_%=;\n\t}" ::"r"(gv_smem_u32(b)),
      "r"(par)
      : "memory");
}
// The weight stream is read once per request and is larger than L2 (VGG FC1:
// 205 MB): it is loaded with an L2 evict-first policy so that it does not
// push co-located tenants' reused weights and activations out of L2.
__device__ __forceinline__ uint64_t gv_evict_first_policy() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ void gv_bulk(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          gv_smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(gv_smem_u32(bar)), "l"(pol)
      : "memory");
}

__device__ __forceinline__ float gv_act(float y, int act) {
  switch (act) {
    case BL_ACT_RELU: return fmaxf(y, 0.f);
    case BL_ACT_RELU6: return fminf(fmaxf(y, 0.f), 6.f);
    case BL_ACT_GELU: return 0.5f * y * (1.f + erff(y * 0.70710678118654752f));
    default: return y;
  }
}

// dot of 16 bf16 weights (two uint4) with 16 bf16 activations at xs
__device__ __forceinline__ float gv_dot16(const uint4& w0, const uint4& w1, const __nv_bfloat16* xs) {
  const uint4 x0 = __ldg(reinterpret_cast<const uint4*>(xs));
  const uint4 x1 = __ldg(reinterpret_cast<const uint4*>(xs) + 1);
  const __nv_bfloat162* a0 = reinterpret_cast<const __nv_bfloat162*>(&w0);
  const __nv_bfloat162* a1 = reinterpret_cast<const __nv_bfloat162*>(&w1);
  const __nv_bfloat162* b0 = reinterpret_cast<const __nv_bfloat162*>(&x0);
  const __nv_bfloat162* b1 = reinterpret_cast<const __nv_bfloat162*>(&x1);
  float s0 = 0.f, s1 = 0.f;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const float2 wa = __bfloat1622float2(a0[j]), xa = __bfloat1622float2(b0[j]);
    const float2 wb = __bfloat1622float2(a1[j]), xb = __bfloat1622float2(b1[j]);
    s0 = fmaf(wa.x, xa.x, s0);
    s0 = fmaf(wa.y, xa.y, s0);
    s1 = fmaf(wb.x, xb.x, s1);
    s1 = fmaf(wb.y, xb.y, s1);
  }
  return s0 + s1;
}

template <int MAXM>
__device__ void gemv_work(const GemvTmaParams& p, const GateArgs& g) {
  extern __shared__ __align__(1024) unsigned char gv_raw[];
  unsigned char* smem = (unsigned char*)(((uintptr_t)gv_raw + 1023) & ~(uintptr_t)1023);
  unsigned char* stage_buf = smem;
  float* red = (float*)(smem + kGvStages * kGvStage);   // [rows][8] row partials
  uint64_t* bars = (uint64_t*)(red + 8 * kGvMaxRows);
  uint64_t* full = bars;                  // [kGvStages]
  uint64_t* empty = bars + kGvStages;     // [kGvStages]
  uint64_t* rfull = empty + kGvStages;    // [2] tile ring
  uint64_t* rempty = rfull + 2;           // [2]
  int* ring = (int*)(rempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kGvStages; ++i) {
      gv_mbar_init(&full[i], 1);
      gv_mbar_init(&empty[i], kGvConsumers);
    }
    for (int i = 0; i < 2; ++i) {
      gv_mbar_init(&rfull[i], 1);
      gv_mbar_init(&rempty[i], kGvConsumers);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  for (int i = threadIdx.x; i < 8 * kGvMaxRows; i += blockDim.x) red[i] = 0.f;
  __syncthreads();
  pdl_wait();
  const long long K = p.K;

  if (warp == 0) {
    if (lane == 0) {
      const uint64_t pol = gv_evict_first_policy();
      bool marked = false;
      int stage = 0, rs = 0;
      uint32_t ph = 0, rph = 0;
      for (;;) {
        const int t = gate_claim(g, marked);
        gv_wait(&rempty[rs], rph ^ 1);
        ring[rs] = t;
        gv_arrive(&rfull[rs]);
        if (++rs == 2) { rs = 0; rph ^= 1; }
        if (t < 0) {
          pdl_trigger();
          break;
        }
        const int n0 = t * p.rows;
        const int nr = min(p.rows, p.N - n0);
        const int kc = kGvElems / p.rows;   // k values per row per stage
        // stage = nr row segments of kc k-values (row r at offset r*kc*2)
        for (long long k0 = 0; k0 < K; k0 += kc) {
          const uint32_t seg = (uint32_t)(min((long long)kc, K - k0) * 2);
          gv_wait(&empty[stage], ph ^ 1);
          gv_expect(&full[stage], seg * nr);
          for (int r = 0; r < nr; ++r)
            gv_bulk(stage_buf + stage * kGvStage + r * (kc * 2), p.W + (size_t)(n0 + r) * K + k0, seg, &full[stage], pol);
          if (++stage == kGvStages) { stage = 0; ph ^= 1; }
        }
      }
    }
  } else {
    const int ctid = (warp - 1) * 32 + lane;   // 0..511
    int stage = 0, rs = 0;
    uint32_t ph = 0, rph = 0;
    for (;;) {
      gv_wait(&rfull[rs], rph);
      const int t = ring[rs];
      __syncwarp();
      if (lane == 0) gv_arrive(&rempty[rs]);
      if (++rs == 2) { rs = 0; rph ^= 1; }
      if (t < 0) break;
      const int n0 = t * p.rows;
      const int nr = min(p.rows, p.N - n0);
      // consumer warp cw owns row cw / wpr of the tile and the 512-k window
      // cw % wpr of every stage (wpr = 16 / rows warps per row): 16
      // consecutive k per lane; the X slice of a stage is shared by all rows
      // through L1
      const int kc = kGvElems / p.rows, wpr = kGvConsumers / p.rows;
      const int row = (warp - 1) / wpr, part = (warp - 1) - row * wpr;
      const int koff = part * kGvWin + lane * kGvRun;
      float acc[MAXM];
#pragma unroll
      for (int m = 0; m < MAXM; ++m) acc[m] = 0.f;
      for (long long k0 = 0; k0 < K; k0 += kc) {
        gv_wait(&full[stage], ph);
        const long long k = k0 + koff;
        if (row < nr && k < K) {
          const uint4* ws = reinterpret_cast<const uint4*>(stage_buf + stage * kGvStage + row * (kc * 2) + koff * 2);
          const uint4 w0 = ws[0], w1 = ws[1];
#pragma unroll
          for (int m = 0; m < MAXM; ++m)
            if (m < p.M) acc[m] += gv_dot16(w0, w1, p.X + (size_t)m * p.ldx + k);
        }
        __syncwarp();
        if (lane == 0) gv_arrive(&empty[stage]);
        if (++stage == kGvStages) { stage = 0; ph ^= 1; }
      }
      if (row < nr) {
#pragma unroll
        for (int m = 0; m < MAXM; ++m) {
          if (m >= p.M) break;
          float v = acc[m];
#pragma unroll
          for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
          if (lane == 0) atomicAdd(&red[row * 8 + m], v);
        }
      }
      asm volatile("bar.sync 1, %0;" ::"n"(32 * kGvConsumers) : "memory");
      if (ctid < p.M * nr) {
        const int r = ctid / p.M, m = ctid - r * p.M;
        float y = red[r * 8 + m];
        red[r * 8 + m] = 0.f;
        const int n = n0 + r;
        if (p.scale) y *= __ldg(p.scale + n);
        if (p.shift) y += __ldg(p.shift + n);
        if (p.R) y += __bfloat162float(p.R[(size_t)m * p.ldr + n]);
        p.Y[(size_t)m * p.ldy + n] = __float2bfloat16_rn(gv_act(y, p.act));
      }
      asm volatile("bar.sync 1, %0;" ::"n"(32 * kGvConsumers) : "memory");
    }
  }
  __syncthreads();
}

template <int MAXM>
__global__ void __launch_bounds__(kGvThreads, 2) k_gemv_tma(const GemvTmaParams p, const GateArgs g) {
  if (gate_in_range(g) || gate_linger(g)) gemv_work<MAXM>(p, g);
  pdl_trigger();
  if (!g.stamp) return;   // light exit
  int last = 0;
  const bool fb = gate_leave(g, last);
  if (fb) gemv_work<MAXM>(p, g);
  if (last) gate_finalize(g, fb);
}
#endif

template <int MAXM>
static cudaError_t launch_gemv_tma(const KernelDesc& d, const GateArgs& g, cudaStream_t st) {
  void* args[2] = {(void*)d.params, (void*)&g};
  return launch_kernel((const void*)k_gemv_tma<MAXM>, dim3(d.grid), dim3(d.block), (size_t)d.smem, st, args);
}

template <int MAXM>
static bool gemv_attr(std::string& err) {
  static std::once_flag once;
  static cudaError_t aerr = cudaSuccess;
  std::call_once(once, [] {
    aerr = cudaFuncSetAttribute((const void*)k_gemv_tma<MAXM>, cudaFuncAttributeMaxDynamicSharedMemorySize, kGvSmem);
  });
  if (aerr != cudaSuccess) err = std::string("gemv attr: ") + cudaGetErrorString(aerr);
  return aerr == cudaSuccess;
}

bool build_gemv_tma(const bl_op& op, const DeviceCaps& caps, KernelDesc& d, std::string& err) {
  err.clear();
  if (op.kind != BL_OP_GEMM || op.dtype != BL_BF16) return false;
  GemvTmaParams p{};
  p.M = (int)op.dims[0];
  p.N = (int)op.dims[1];
  p.K = (int)op.dims[2];
  p.ldx = op.dims[3] ? (int)op.dims[3] : p.K;
  p.ldy = op.dims[4] ? (int)op.dims[4] : p.N;
  p.ldr = op.dims[5] ? (int)op.dims[5] : p.N;
  if (p.M < 1 || p.M > 8 || p.N < 1 || p.K % kGvRun || p.ldx % 8) return false;
  p.X = (const __nv_bfloat16*)op.ptr[0];
  p.W = (const __nv_bfloat16*)op.ptr[1];
  if ((((uintptr_t)p.X) | ((uintptr_t)p.W)) & 15) return false;
  p.scale = (const float*)op.ptr[2];
  p.shift = (const float*)op.ptr[3];
  p.R = (const __nv_bfloat16*)op.ptr[4];
  p.Y = (__nv_bfloat16*)op.ptr[5];
  p.act = op.act;
  p.invK = 1.0f / (float)p.K;
  p.warp_rows = (p.K % (32 * kGvRun)) == 0;
  // rows per tile: 4 (measured on B200, profiles/round1/gemv_rows.txt: VGG FC1
  // 25088->4096 rows 8/4/2/1 = 52.0/40.7/46.8/53.7 us -- 8-row tiles (400 KB)
  // leave a long tail in the dynamic queue, 1-2-row tiles pay the per-tile
  // fold too often), fewer when that leaves under one tile per SM.  Three
  // other schedules were measured and dropped: a flat weight stream whose
  // 16-64 KB tiles cut rows (fp32 row sums completed through a global k
  // counter: half the bandwidth -- the gpu-scope fences also invalidate L1
  // and the X reloads), guided tile heights 4 -> 2 -> 1 (10% slower: partial
  // stages), and the last wave's row tiles cut into K halves joined by fp32
  // atomics (18% slower); profiles/round1/gemv_{stream_sweep,guided_ab,
  // split_tail_ab}.txt
  int rows = 4;
  while (rows > 1 && (long long)((p.N + rows - 1) / rows) < caps.S) rows /= 2;
  if (const char* e = std::getenv("BLESS_GEMV_ROWS")) rows = std::atoi(e);
  if (rows != 1 && rows != 2 && rows != 4 && rows != 8) rows = kGvMaxRows;
  p.rows = rows;
  const bool m1 = p.M == 1;
  if (!(m1 ? gemv_attr<1>(err) : gemv_attr<8>(err))) return false;
  d.op = op;
  d.tiles = (uint32_t)((p.N + rows - 1) / rows);
  d.grid = 2 * caps.S;   // two CTAs (two independent TMA streams) per SM
  d.block = kGvThreads;
  d.smem = kGvSmem;
  d.launch = m1 ? launch_gemv_tma<1> : launch_gemv_tma<8>;
  d.kernel_fn = m1 ? (const void*)k_gemv_tma<1> : (const void*)k_gemv_tma<8>;
  d.family = "gemv_tma_bf16";
  d.flops = 2.0 * p.M * p.N * p.K;
  d.bytes = 2.0 * ((double)p.N * p.K + (double)p.M * p.K + (double)p.M * p.N);
  std::memcpy(d.params, &p, sizeof(p));
  return true;
}

}  // namespace bless
