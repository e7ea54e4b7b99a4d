// attn_tc.cu -- fused scaled-dot-product attention on the 5th-generation tensor
// cores for the BERT tenants (L <= 512, L % 128 == 0, dh = 64,
// all-ones mask).  One work tile = (head, 128-query block):
//
//   1. TMA: Q block [128 x 64] and K [L x 64] of the head (K-major, SW128);
//   2. tcgen05.mma: S = Q K^T into TMEM (fp32, L <= 512 columns; N <= 256 per
//      instruction);
//   3. 4 softmax warps (thread = query row): tcgen05.ld the row twice (max,
//      then exp/sum), write P = exp(S*scale - max) as bf16 into shared memory
//      in the UMMA K-major SW128 layout;  meanwhile TMA loads V [L x 64] into
//      the freed Q/K buffer -- V as stored (keys x dh) is the canonical
//      MN-major layout of the B operand, so no transpose is needed;
//   4. tcgen05.mma: O = P V into TMEM (64 columns);
//   5. epilogue: O / rowsum -> bf16 -> out[q, h*64 : h*64 + 64].
// Warp 0: TMA producer + MMA issuer (one thread); warps 1..8: softmax and
// epilogue, four warps per TMEM lane quarter (quarter = warp % 4), each taking
// one quarter of the keys (and of O's columns); the row max and row sum of the
// parts meet in shared memory.  (With one warp per quarter the softmax
// was the serial part of a BERT-large tile: 16.6 us per launch.)  Under the
// SM-gated executor.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "../runtime/kdesc.hpp"
#include "executor.cuh"

namespace bless {

struct AttnTcParams {
  CUtensorMap tm;  // QKV [L rows, 3*H*dh cols], box {64, 128}, SW128
  __nv_bfloat16* O;
  int L, H, dh, ldo, qblocks;
  float scale_log2e;  // scale * log2(e)
};

namespace attn {
constexpr int kParts = 4;                 // key parts per TMEM lane quarter
constexpr int kSoftWarps = 4 * kParts;    // softmax/epilogue warps
constexpr int kThreads = 32 + 32 * kSoftWarps;   // warp 0 producer/MMA, warps 1-8 softmax/epilogue
constexpr int kMaxL = 384;                // S (L fp32 columns) + O (64 columns at 448) fit in 512 TMEM columns
constexpr int kQBytes = 128 * 128;        // 128 rows x 128 B
constexpr int kKVBytes = kMaxL * 128;     // L rows x 128 B (K, later V)
constexpr int kPBytes = (kMaxL / 64) * 128 * 128;  // L/64 K-blocks of [128 rows x 128 B]
constexpr int kSmem = kQBytes + kKVBytes + kPBytes + 1024 + 256 + 2 * kParts * 128 * 4;   // + row max/sum parts
}  // namespace attn

#ifdef __CUDACC__
namespace attn {
__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void bar_init(uint64_t* b, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(c));
}
__device__ __forceinline__ void bar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void bar_expect(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bar_wait(uint64_t* b, uint32_t par) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tW_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra W_%=;\n\t}" ::"r"(su32(b)),
      "r"(par)
      : "memory");
}
__device__ __forceinline__ void tma2d(void* dst, const CUtensorMap* m, uint64_t* bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
          su32(dst)),
      "l"(m), "r"(su32(bar)), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc)
      : "memory");
}
__device__ __forceinline__ void commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(bar))
               : "memory");
}
// Elected-lane variants: warp 0 runs the load/MMA sequence as a whole warp
// (uniform descriptors in uniform registers) and one elected lane issues
// (issuing under `if (lane == 0)` wrapped every tcgen05.mma in an ELECT +
// R2UR.BROADCAST waterfall loop -- see tc_gemm.cu).
__device__ __forceinline__ void bar_expect_e(uint64_t* b, uint32_t bytes) {
  asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
               "@e mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n\t}" ::"r"(su32(b)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void tma2d_e(void* dst, const CUtensorMap* m, uint64_t* bar, int c0, int c1) {
  asm volatile(
      "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
      "@e cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
      "\n\t}" ::"r"(su32(dst)),
      "l"(m), "r"(su32(bar)), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void mma_e(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p, e;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc)
      : "memory");
}
__device__ __forceinline__ void commit_e(uint64_t* bar) {
  asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
               "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(bar))
               : "memory");
}
__device__ __forceinline__ void ld16(uint32_t taddr, uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),
        "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
// K-major SW128 (rows of 128 B, 8-row atoms of 1024 B)
__device__ __forceinline__ uint64_t desc_k(uint32_t saddr) {
  uint64_t d = (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;                   // LBO (unused for swizzled K-major)
  d |= (uint64_t)(1024 >> 4) << 32;         // SBO: 8 rows x 128 B
  d |= (uint64_t)1 << 46;                   // version (tcgen05)
  d |= (uint64_t)2 << 61;                   // SWIZZLE_128B
  return d;
}
// MN-major SW128 B operand (N = 64 = one 128-B atom row per K index; 8-K-row
// groups 1024 B apart): LBO = stride between N atoms (only one here), SBO =
// stride between 8-row K groups.
__device__ __forceinline__ uint64_t desc_mn(uint32_t saddr) {
  uint64_t d = (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)(8192 >> 4) << 16;         // LBO
  d |= (uint64_t)(1024 >> 4) << 32;         // SBO
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}
// kind::f16, bf16 x bf16 -> f32, M = 128; b_mn: B operand MN-major
__device__ __forceinline__ uint32_t idesc(int N, bool b_mn) {
  uint32_t d = (1u << 4) | (1u << 7) | (1u << 10);
  if (b_mn) d |= 1u << 16;
  d |= (uint32_t)(N >> 3) << 17;
  d |= (uint32_t)(128 >> 4) << 24;
  return d;
}
}  // namespace attn

__device__ void attn_work(const AttnTcParams& p, const GateArgs& g) {
  using namespace attn;
  extern __shared__ __align__(1024) unsigned char a_raw[];
  unsigned char* smem = (unsigned char*)(((uintptr_t)a_raw + 1023) & ~(uintptr_t)1023);
  unsigned char* sQ = smem;
  unsigned char* sKV = smem + kQBytes;
  unsigned char* sP = sKV + kKVBytes;
  uint64_t* bars = (uint64_t*)(sP + kPBytes);
  uint64_t* b_qk = bars;       // Q and K landed
  uint64_t* b_v = bars + 1;    // V landed
  uint64_t* b_s = bars + 2;    // S ready (MMA commit)
  uint64_t* b_p = bars + 3;    // P written (4 softmax warps)
  uint64_t* b_o = bars + 4;    // O ready (MMA commit)
  uint64_t* b_done = bars + 5; // epilogue finished reading TMEM (4 warps)
  uint64_t* b_p2 = bars + 6;   // P_lo written (4 softmax warps)
  uint64_t* b_o1 = bars + 7;   // P_hi MMAs done (MMA commit)
  int* tile_slot = (int*)(bars + 8);
  uint32_t* tmem_slot = (uint32_t*)(tile_slot + 1);
  float* red_max = (float*)(bars + 32);   // [kParts][128] per key part
  float* red_sum = red_max + kParts * 128;  // [kParts][128]
  const int warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0), lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    bar_init(b_qk, 1);
    bar_init(b_v, 1);
    bar_init(b_s, 1);
    bar_init(b_p, kSoftWarps);
    bar_init(b_o, 1);
    bar_init(b_done, kSoftWarps);
    bar_init(b_p2, kSoftWarps);
    bar_init(b_o1, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(tmem_slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = __shfl_sync(0xffffffffu, *tmem_slot, 0);
  pdl_wait();
  const int L = p.L, H = p.H;
  const int nkb = L / 64;      // 64-key blocks
  bool marked = false;
  uint32_t ph = 0;
  for (;;) {
    if (threadIdx.x == 0) *tile_slot = gate_claim(g, marked);
    __syncthreads();
    const int t = __shfl_sync(0xffffffffu, *tile_slot, 0);
    __syncthreads();
    if (t < 0) break;
    const int h = t / p.qblocks, qb = t - h * p.qblocks;
    if (warp == 0) {
      // whole warp: loads / MMAs issued by one elected lane (uniform loop)
      // ---- loads: Q block and K (K-major, SW128)
      bar_expect_e(b_qk, kQBytes + L * 128);
      tma2d_e(sQ, &p.tm, b_qk, h * 64, qb * 128);
      for (int r = 0; r < L; r += 128) tma2d_e(sKV + r * 128, &p.tm, b_qk, H * 64 + h * 64, r);
      bar_wait(b_qk, ph);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      // ---- S = Q K^T  (N chunks of <= 256 keys, 4 k-steps of 16 over dh = 64)
      for (int n0 = 0; n0 < L; n0 += 256) {
        const int N = (L - n0) < 256 ? (L - n0) : 256;
        const uint32_t id = idesc(N, false);
        for (int k = 0; k < 4; ++k)
          mma_e(tmem + n0, desc_k(su32(sQ) + k * 32), desc_k(su32(sKV) + n0 * 128 + k * 32), id, k ? 1u : 0u);
      }
      commit_e(b_s);
      // ---- V into the K buffer once the S MMAs have consumed it
      bar_wait(b_s, ph);
      bar_expect_e(b_v, L * 128);
      for (int r = 0; r < L; r += 128) tma2d_e(sKV + r * 128, &p.tm, b_v, 2 * H * 64 + h * 64, r);
      bar_wait(b_v, ph);
      // ---- O = P V : A = P (K-major, nkb blocks of 64 keys), B = V (MN-major, keys x dh),
      // in two passes P = P_hi + P_lo (bf16 each) for ~16-bit precision of P
      const uint32_t id = idesc(64, true);
      for (int pass = 0; pass < 2; ++pass) {
        bar_wait(pass == 0 ? b_p : b_p2, ph);   // P part in smem (writers fenced the generic proxy)
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        for (int kb = 0; kb < nkb; ++kb)
          for (int k = 0; k < 4; ++k)
            mma_e(tmem + 448, desc_k(su32(sP) + kb * 16384 + k * 32),
                  desc_mn(su32(sKV) + kb * 64 * 128 + k * 16 * 128), id, (pass | kb | k) ? 1u : 0u);
        commit_e(pass == 0 ? b_o1 : b_o);
      }
      bar_wait(b_done, ph);   // epilogue drained O before the next tile reuses TMEM / smem
      __syncwarp();
    } else {
      // ---- softmax: thread = query row (TMEM lane) x key half
      const int q = warp & 3;
      const int part = (warp - 1) >> 2;
      const int row = q * 32 + lane;
      const int c0 = part * (L / kParts), c1 = c0 + L / kParts;   // L % 128 == 0: parts are whole 16-key chunks
      const uint32_t trow = tmem + ((uint32_t)(q * 32) << 16);
      bar_wait(b_s, ph);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      float mx = -INFINITY;
      for (int c = c0; c < c1; c += 16) {
        uint32_t v[16];
        ld16(trow + c, v);
#pragma unroll
        for (int i = 0; i < 16; ++i) mx = fmaxf(mx, __uint_as_float(v[i]));
      }
      red_max[part * 128 + row] = mx;
      asm volatile("bar.sync 1, %0;" ::"n"(32 * kSoftWarps) : "memory");   // every part's maximum
#pragma unroll
      for (int i = 0; i < kParts; ++i) mx = fmaxf(mx, red_max[i * 128 + row]);
      const float moff = mx * p.scale_log2e;
      float sum = 0.f;
      const int rr = row & 7;
      unsigned char* prow = sP + (row >> 3) * 1024 + rr * 128;
      // pass 0 writes P_hi = bf16(e), pass 1 writes P_lo = bf16(e - P_hi)
      for (int pass = 0; pass < 2; ++pass) {
        if (pass == 1) bar_wait(b_o1, ph);   // the P_hi MMAs have consumed the buffer
        for (int c = c0; c < c1; c += 16) {
          uint32_t v[16];
          ld16(trow + c, v);
          uint32_t pk[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            float e0 = exp2f(fmaf(__uint_as_float(v[2 * i]), p.scale_log2e, -moff));
            float e1 = exp2f(fmaf(__uint_as_float(v[2 * i + 1]), p.scale_log2e, -moff));
            if (pass == 0) {
              sum += e0 + e1;
            } else {
              const float2 hi = __bfloat1622float2(__floats2bfloat162_rn(e0, e1));
              e0 -= hi.x;
              e1 -= hi.y;
            }
            const __nv_bfloat162 b2 = __floats2bfloat162_rn(e0, e1);
            pk[i] = *reinterpret_cast<const uint32_t*>(&b2);
          }
          // keys c..c+15 -> K-block c/64, 16-byte chunks (c%64)/8 and +1, SW128 swizzle by row%8
          unsigned char* blk = prow + (c >> 6) * 16384;
          const int ch = (c & 63) >> 3;
          *reinterpret_cast<uint4*>(blk + ((ch ^ rr) << 4)) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
          *reinterpret_cast<uint4*>(blk + (((ch + 1) ^ rr) << 4)) = make_uint4(pk[4], pk[5], pk[6], pk[7]);
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // P visible to the tensor core
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncwarp();
        if (lane == 0) bar_arrive(pass == 0 ? b_p : b_p2);
      }
      red_sum[part * 128 + row] = sum;
      // ---- epilogue (this warp: O columns [16 * part, 16 * part + 16))
      bar_wait(b_o, ph);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      asm volatile("bar.sync 1, %0;" ::"n"(32 * kSoftWarps) : "memory");   // every part's sum
      float tot = 0.f;
#pragma unroll
      for (int i = 0; i < kParts; ++i) tot += red_sum[i * 128 + row];
      const float inv = 1.f / tot;
      const int qrow = qb * 128 + row;
      __nv_bfloat16* out = p.O + (size_t)qrow * p.ldo + h * 64;
#pragma unroll 1
      for (int c = 16 * part; c < 16 * part + 16; c += 16) {
        uint32_t v[16];
        ld16(trow + 448 + c, v);
        uint32_t pk[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const __nv_bfloat162 b2 =
              __floats2bfloat162_rn(__uint_as_float(v[2 * i]) * inv, __uint_as_float(v[2 * i + 1]) * inv);
          pk[i] = *reinterpret_cast<const uint32_t*>(&b2);
        }
        *reinterpret_cast<uint4*>(out + c) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
        *reinterpret_cast<uint4*>(out + c + 8) = make_uint4(pk[4], pk[5], pk[6], pk[7]);
      }
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      __syncwarp();
      if (lane == 0) bar_arrive(b_done);
    }
    ph ^= 1;
  }
  pdl_trigger();
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
  __syncthreads();
}

__global__ void __launch_bounds__(attn::kThreads, 1) k_attn_tc(const __grid_constant__ AttnTcParams p,
                                                                const GateArgs g) {
  if (gate_in_range(g) || gate_linger(g)) attn_work(p, g);
  pdl_trigger();
  if (!g.stamp) return;   // light exit
  int last = 0;
  const bool fb = gate_leave(g, last);
  if (fb) attn_work(p, g);
  if (last) gate_finalize(g, fb);
}
#endif

static cudaError_t launch_attn_tc(const KernelDesc& d, const GateArgs& g, cudaStream_t st) {
  void* args[2] = {(void*)d.params, (void*)&g};
  return launch_kernel((const void*)k_attn_tc, dim3(d.grid), dim3(d.block), (size_t)d.smem, st, args);
}

typedef CUresult (*EncodeTiledFn2)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

bool build_attn_tc(const bl_op& op, const DeviceCaps& caps, KernelDesc& d, std::string& err) {
  err.clear();
  if (op.kind != BL_OP_ATTENTION || op.dtype != BL_BF16 || caps.cc_major != 10) return false;
  if (std::getenv("BLESS_ATTN_SIMT")) return false;
  AttnTcParams p;
  std::memset(&p, 0, sizeof(p));
  p.L = (int)op.dims[0];
  p.H = (int)op.dims[1];
  p.dh = (int)op.dims[2];
  const int ldq = op.dims[3] ? (int)op.dims[3] : 3 * p.H * p.dh;
  p.ldo = op.dims[4] ? (int)op.dims[4] : p.H * p.dh;
  if (p.dh != 64 || p.L % 128 || p.L > attn::kMaxL || ldq != 3 * p.H * 64 || p.ldo % 8) return false;
  const void* qkv = op.ptr[0];
  p.O = (__nv_bfloat16*)op.ptr[1];
  if ((((uintptr_t)qkv) | ((uintptr_t)p.O)) & 15) return false;
  const float scale = op.fparam[0] != 0.f ? op.fparam[0] : 1.0f / sqrtf(64.f);
  p.scale_log2e = scale * 1.4426950408889634f;
  p.qblocks = p.L / 128;
  static EncodeTiledFn2 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (EncodeTiledFn2)f;
    cudaFuncSetAttribute((const void*)k_attn_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, attn::kSmem);
  });
  if (!fn) { err = "cuTensorMapEncodeTiled unavailable"; return false; }
  cuuint64_t dims[2] = {(cuuint64_t)ldq, (cuuint64_t)p.L};
  cuuint64_t strides[1] = {(cuuint64_t)ldq * 2};
  cuuint32_t box[2] = {64, 128};
  cuuint32_t es[2] = {1, 1};
  if (fn(&p.tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(qkv), dims, strides, box, es,
         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
    err = "attention tensor map";
    return false;
  }
  d.op = op;
  d.tiles = (uint32_t)(p.H * p.qblocks);
  d.block = attn::kThreads;
  d.grid = caps.S;
  d.smem = attn::kSmem;
  d.launch = launch_attn_tc;
  d.kernel_fn = (const void*)k_attn_tc;
  d.family = "attention_tc_bf16";
  d.flops = 4.0 * p.H * (double)p.L * p.L * 64;
  d.bytes = 2.0 * p.L * (3.0 * p.H * 64 + p.H * 64);
  static_assert(sizeof(AttnTcParams) <= sizeof(d.params), "params");
  std::memcpy(d.params, &p, sizeof(p));
  return true;
}

}  // namespace bless
