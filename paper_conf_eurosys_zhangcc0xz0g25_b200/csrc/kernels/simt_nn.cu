// simt_nn.cu -- CUDA-core tenant kernels for configs C3/C4 under the SM-gated
// executor: LayerNorm (+ residual), scaled
// dot-product attention, BERT embedding (gather + add + LN), depthwise conv
// (MobileNetV2), strided per-channel affine + activation (DenseNet BN-ReLU on
// a channel slice of the concat buffer).  bf16 storage, fp32 math; semantics
// as oracle/layers_ref.py.  None of these is a dense contraction worth the
// tensor cores at the configs' sizes except attention: L % 128 == 0 runs on
// the fused tcgen05 kernel (attn_tc.cu); the CUDA-core attention here covers
// the other sequence lengths (and BLESS_ATTN_SIMT=1).
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>

#include "../runtime/kdesc.hpp"
#include "executor.cuh"

namespace bless {
namespace nn {

typedef __nv_bfloat16 bf16;

__device__ __forceinline__ float act_f(float y, int act) {
  switch (act) {
    case BL_ACT_RELU: return fmaxf(y, 0.f);
    case BL_ACT_RELU6: return fminf(fmaxf(y, 0.f), 6.f);
    case BL_ACT_GELU: return 0.5f * y * (1.f + erff(y * 0.70710678118654752f));
    default: return y;
  }
}
__device__ __forceinline__ void ld8(const bf16* p, float (&f)[8]) {
  const uint4 u = *reinterpret_cast<const uint4*>(p);
  const __nv_bfloat162* b = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const float2 v = __bfloat1622float2(b[i]);
    f[2 * i] = v.x;
    f[2 * i + 1] = v.y;
  }
}
__device__ __forceinline__ void st8(bf16* p, const float (&f)[8]) {
  uint4 u;
  __nv_bfloat162* b = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
  for (int i = 0; i < 4; ++i) b[i] = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
  *reinterpret_cast<uint4*>(p) = u;
}
__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// ---------------------------------------------------------------------------
// LayerNorm / Embedding: one warp per row, C = 256 * V (V <= 4 vectors of 8 per lane)
// ---------------------------------------------------------------------------
struct LnParams {
  const bf16* X;
  const float* gamma;
  const float* beta;
  const bf16* R;
  bf16* Y;
  int rows, C, ldx, ldy;
  float eps;
  // embedding
  const int* ids;
  const bf16* word;
  const bf16* pos;
  const bf16* type;
  int embed;
};
constexpr int kLnMaxVec = 4;   // C <= 1024

struct LayerNorm {
  using Params = LnParams;
  __device__ static void tile(const Params& p, int t, unsigned char*) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int row = t * 8 + warp;
    if (row >= p.rows) return;
    const int nv = p.C / 256;
    float x[kLnMaxVec][8];
    float s = 0.f;
#pragma unroll
    for (int v = 0; v < kLnMaxVec; ++v) {
      if (v >= nv) break;
      const int c = (v * 32 + lane) * 8;
      if (p.embed) {
        float a[8], b[8], e[8];
        const int id = __ldg(p.ids + row);
        ld8(p.word + (size_t)id * p.C + c, a);
        ld8(p.pos + (size_t)row * p.C + c, b);
        ld8(p.type + c, e);
#pragma unroll
        for (int i = 0; i < 8; ++i) x[v][i] = a[i] + b[i] + e[i];
      } else {
        ld8(p.X + (size_t)row * p.ldx + c, x[v]);
        if (p.R) {
          float r[8];
          ld8(p.R + (size_t)row * p.ldx + c, r);
#pragma unroll
          for (int i = 0; i < 8; ++i) x[v][i] += r[i];
        }
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) s += x[v][i];
    }
    const float mean = warp_sum(s) / (float)p.C;
    float q = 0.f;
#pragma unroll
    for (int v = 0; v < kLnMaxVec; ++v) {
      if (v >= nv) break;
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const float d = x[v][i] - mean;
        q += d * d;
      }
    }
    const float rstd = rsqrtf(warp_sum(q) / (float)p.C + p.eps);
#pragma unroll
    for (int v = 0; v < kLnMaxVec; ++v) {
      if (v >= nv) break;
      const int c = (v * 32 + lane) * 8;
      float y[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) y[i] = (x[v][i] - mean) * rstd * __ldg(p.gamma + c + i) + __ldg(p.beta + c + i);
      st8(p.Y + (size_t)row * p.ldy + c, y);
    }
  }
};

// ---------------------------------------------------------------------------
// Attention: tile = (head, 16 queries); K, V of the head staged in smem (row
// stride padded to 66 elements: conflict-free column reads); one warp per
// query: lanes own keys j = lane + 32 i for the scores, output dims 2 lane,
// 2 lane + 1 for P V; softmax with warp reductions (max-subtracted, fp32).
// ---------------------------------------------------------------------------
struct AttnParams {
  const bf16* qkv;
  bf16* o;
  int L, H, dh, ldq, ldo, qtiles;
  float scale;
};
constexpr int kAttnQB = 16;
constexpr int kAttnMaxL = 512;
constexpr int kAttnKs = 66;   // padded K/V row stride (elements)

struct Attention {
  using Params = AttnParams;
  __device__ static void tile(const Params& p, int t, unsigned char* smem) {
    const int h = t / p.qtiles, q0 = (t - h * p.qtiles) * kAttnQB;
    bf16* Ks = reinterpret_cast<bf16*>(smem);
    bf16* Vs = Ks + (size_t)p.L * kAttnKs;
    float* qs = reinterpret_cast<float*>(Vs + (size_t)p.L * kAttnKs);   // [8 warps][64]
    const int hd = p.H * p.dh;
    // stage K and V (64-element rows, 8 x 16 B each)
    for (int i = threadIdx.x; i < p.L * 8; i += blockDim.x) {
      const int r = i >> 3, v = i & 7;
      const bf16* src = p.qkv + (size_t)r * p.ldq + h * p.dh + v * 8;
      const uint4 kk = *reinterpret_cast<const uint4*>(src + hd);
      const uint4 vv = *reinterpret_cast<const uint4*>(src + 2 * hd);
      uint32_t* kd = reinterpret_cast<uint32_t*>(Ks + (size_t)r * kAttnKs + v * 8);
      uint32_t* vd = reinterpret_cast<uint32_t*>(Vs + (size_t)r * kAttnKs + v * 8);
      kd[0] = kk.x; kd[1] = kk.y; kd[2] = kk.z; kd[3] = kk.w;
      vd[0] = vv.x; vd[1] = vv.y; vd[2] = vv.z; vd[3] = vv.w;
    }
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    float* q = qs + warp * 64;
    for (int qi = warp; qi < kAttnQB; qi += blockDim.x >> 5) {
      const int qt = q0 + qi;
      if (qt >= p.L) break;
      {
        const bf16* qsrc = p.qkv + (size_t)qt * p.ldq + h * p.dh;
        const float2 f = __bfloat1622float2(reinterpret_cast<const __nv_bfloat162*>(qsrc)[lane]);
        q[2 * lane] = f.x * p.scale;
        q[2 * lane + 1] = f.y * p.scale;
      }
      __syncwarp();
      float sc[kAttnMaxL / 32];
      float mx = -INFINITY;
#pragma unroll
      for (int i = 0; i < kAttnMaxL / 32; ++i) {
        const int j = i * 32 + lane;
        float s = -INFINITY;
        if (j < p.L) {
          const __nv_bfloat162* kr = reinterpret_cast<const __nv_bfloat162*>(Ks + (size_t)j * kAttnKs);
          s = 0.f;
#pragma unroll 8
          for (int d = 0; d < 32; ++d) {
            const float2 kv = __bfloat1622float2(kr[d]);
            s = fmaf(q[2 * d], kv.x, s);
            s = fmaf(q[2 * d + 1], kv.y, s);
          }
        }
        sc[i] = s;
        mx = fmaxf(mx, s);
      }
      mx = warp_max(mx);
      float sum = 0.f;
#pragma unroll
      for (int i = 0; i < kAttnMaxL / 32; ++i) {
        const float e = (i * 32 + lane < p.L) ? __expf(sc[i] - mx) : 0.f;
        sc[i] = e;
        sum += e;
      }
      sum = warp_sum(sum);
      float a0 = 0.f, a1 = 0.f;
#pragma unroll
      for (int i = 0; i < kAttnMaxL / 32; ++i) {
        if (i * 32 >= p.L) break;
        for (int l = 0; l < 32; ++l) {
          const int j = i * 32 + l;
          if (j >= p.L) break;
          const float pj = __shfl_sync(0xffffffffu, sc[i], l);
          const float2 vv = __bfloat1622float2(reinterpret_cast<const __nv_bfloat162*>(Vs + (size_t)j * kAttnKs)[lane]);
          a0 = fmaf(pj, vv.x, a0);
          a1 = fmaf(pj, vv.y, a1);
        }
      }
      const float inv = 1.f / sum;
      reinterpret_cast<__nv_bfloat162*>(p.o + (size_t)qt * p.ldo + h * p.dh)[lane] =
          __floats2bfloat162_rn(a0 * inv, a1 * inv);
      __syncwarp();
    }
    __syncthreads();   // K/V smem reused by the next tile of this CTA
  }
};

// ---------------------------------------------------------------------------
// Depthwise conv: one thread per (output pixel, 8 channels)
// ---------------------------------------------------------------------------
struct DwParams {
  const bf16* X;
  const bf16* W;   // [C][R][S]
  const float* scale;
  const float* shift;
  const bf16* R;
  bf16* Y;
  int H, Wd, C, R_, S_, stride, pad, OH, OW, act;
  long long items;
  int per_tile;
};

struct DwConv {
  using Params = DwParams;
  __device__ static void tile(const Params& p, int t, unsigned char*) {
    const int CV = p.C / 8;
    const long long i0 = (long long)t * p.per_tile, i1 = min(i0 + p.per_tile, p.items);
    for (long long it = i0 + threadIdx.x; it < i1; it += blockDim.x) {
      const int cv = (int)(it % CV);
      const int pix = (int)(it / CV);
      const int oh = pix / p.OW, ow = pix - oh * p.OW;
      float acc[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] = 0.f;
      const int c0 = cv * 8;
      for (int r = 0; r < p.R_; ++r) {
        const int ih = oh * p.stride - p.pad + r;
        if (ih < 0 || ih >= p.H) continue;
        for (int s = 0; s < p.S_; ++s) {
          const int iw = ow * p.stride - p.pad + s;
          if (iw < 0 || iw >= p.Wd) continue;
          float x[8];
          ld8(p.X + ((size_t)ih * p.Wd + iw) * p.C + c0, x);
#pragma unroll
          for (int i = 0; i < 8; ++i)
            acc[i] = fmaf(x[i], __bfloat162float(p.W[((size_t)(c0 + i) * p.R_ + r) * p.S_ + s]), acc[i]);
        }
      }
      float res[8];
      if (p.R) ld8(p.R + (size_t)pix * p.C + c0, res);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        float y = acc[i];
        if (p.scale) y *= __ldg(p.scale + c0 + i);
        if (p.shift) y += __ldg(p.shift + c0 + i);
        if (p.R) y += res[i];
        acc[i] = act_f(y, p.act);
      }
      st8(p.Y + (size_t)pix * p.C + c0, acc);
    }
  }
};

// ---------------------------------------------------------------------------
// Strided eltwise: Y[r, c] = act(X[r, c] * scale[c] + shift[c] (+ R[r, c]))
// ---------------------------------------------------------------------------
struct EwParams {
  const bf16* X;
  const float* scale;
  const float* shift;
  const bf16* R;
  bf16* Y;
  int rows, C, ldx, ldy, act;
  long long items;
  int per_tile;
};

struct Eltwise {
  using Params = EwParams;
  __device__ static void tile(const Params& p, int t, unsigned char*) {
    const int CV = p.C / 8;
    const long long i0 = (long long)t * p.per_tile, i1 = min(i0 + p.per_tile, p.items);
    for (long long it = i0 + threadIdx.x; it < i1; it += blockDim.x) {
      const int cv = (int)(it % CV);
      const int r = (int)(it / CV);
      const int c0 = cv * 8;
      float x[8], rr[8];
      ld8(p.X + (size_t)r * p.ldx + c0, x);
      if (p.R) ld8(p.R + (size_t)r * p.ldy + c0, rr);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        float y = x[i];
        if (p.scale) y *= __ldg(p.scale + c0 + i);
        if (p.shift) y += __ldg(p.shift + c0 + i);
        if (p.R) y += rr[i];
        x[i] = act_f(y, p.act);
      }
      st8(p.Y + (size_t)r * p.ldy + c0, x);
    }
  }
};

template <class Op>
__global__ void __launch_bounds__(256) k_nn(const typename Op::Params p, const GateArgs g) {
  extern __shared__ __align__(16) unsigned char smem[];
  gated_run<Op>(p, g, smem);
}

template <class Op>
static cudaError_t launch_nn(const KernelDesc& d, const GateArgs& g, cudaStream_t st) {
  void* args[2] = {(void*)d.params, (void*)&g};
  return launch_kernel((const void*)k_nn<Op>, dim3(launch_grid(d, g)), dim3(d.block), (size_t)d.smem, st, args);
}

template <class Op>
static void use_nn(KernelDesc& d) {
  d.launch = launch_nn<Op>;
  d.kernel_fn = (const void*)k_nn<Op>;
}

static bool aligned16(const void* p) { return (((uintptr_t)p) & 15) == 0; }

}  // namespace nn

bool build_nn(const bl_op& op, const DeviceCaps& caps, KernelDesc& d, std::string& err) {
  using namespace nn;
  err.clear();
  const int k = op.kind;
  if (k != BL_OP_LAYERNORM && k != BL_OP_ATTENTION && k != BL_OP_EMBED && k != BL_OP_DWCONV && k != BL_OP_ELTWISE)
    return false;
  if (op.dtype != BL_BF16) return false;   // fp32 eltwise stays on the generic path
  d.op = op;
  d.block = 256;
  d.grid = caps.S * 2;
  d.smem = 0;
  if (k == BL_OP_LAYERNORM || k == BL_OP_EMBED) {
    LnParams p{};
    p.embed = k == BL_OP_EMBED;
    p.rows = (int)op.dims[0];
    p.C = (int)op.dims[1];
    p.eps = op.fparam[0] != 0.f ? op.fparam[0] : 1e-12f;
    if (p.embed) {
      p.ids = (const int*)op.ptr[0];
      p.word = (const bf16*)op.ptr[1];
      p.pos = (const bf16*)op.ptr[2];
      p.type = (const bf16*)op.ptr[3];
      p.gamma = (const float*)op.ptr[4];
      p.beta = (const float*)op.ptr[5];
      p.Y = (bf16*)op.ptr[6];
      p.ldx = p.ldy = p.C;
    } else {
      p.X = (const bf16*)op.ptr[0];
      p.gamma = (const float*)op.ptr[1];
      p.beta = (const float*)op.ptr[2];
      p.R = (const bf16*)op.ptr[3];
      p.Y = (bf16*)op.ptr[4];
      p.ldx = op.dims[2] ? (int)op.dims[2] : p.C;
      p.ldy = op.dims[3] ? (int)op.dims[3] : p.C;
    }
    if (p.rows < 1 || p.C % 256 || p.C > 256 * kLnMaxVec || p.ldx % 8 || p.ldy % 8 || !p.gamma || !p.beta) {
      err = "layernorm: C must be a multiple of 256 and <= 1024";
      return false;
    }
    d.tiles = (uint32_t)((p.rows + 7) / 8);
    std::memcpy(d.params, &p, sizeof(p));
    use_nn<LayerNorm>(d);
    d.family = p.embed ? "embed_ln_bf16" : "layernorm_bf16";
    d.max_occ = 1;   // B200 sweep: fastest with 1 CTA/SM (profiles/round1/occ_cap.txt)
    d.bytes = 2.0 * p.rows * p.C * (p.R ? 3 : 2);
    return true;
  }
  if (k == BL_OP_ATTENTION) {
    AttnParams p{};
    p.qkv = (const bf16*)op.ptr[0];
    p.o = (bf16*)op.ptr[1];
    p.L = (int)op.dims[0];
    p.H = (int)op.dims[1];
    p.dh = (int)op.dims[2];
    p.ldq = op.dims[3] ? (int)op.dims[3] : 3 * p.H * p.dh;
    p.ldo = op.dims[4] ? (int)op.dims[4] : p.H * p.dh;
    p.scale = op.fparam[0] != 0.f ? op.fparam[0] : 1.0f / sqrtf((float)p.dh);
    if (p.L < 1 || p.L > kAttnMaxL || p.dh != 64 || p.H < 1 || p.ldq % 8 || p.ldo % 2 || !aligned16(p.qkv)) {
      err = "attention: dh must be 64, L <= 512";
      return false;
    }
    p.qtiles = (p.L + kAttnQB - 1) / kAttnQB;
    d.tiles = (uint32_t)(p.H * p.qtiles);
    d.smem = 2 * p.L * kAttnKs * 2 + 8 * 64 * 4;
    if (d.smem > 48 * 1024 &&
        cudaFuncSetAttribute((const void*)k_nn<Attention>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             2 * kAttnMaxL * kAttnKs * 2 + 8 * 64 * 4) != cudaSuccess) {
      err = "attention smem attribute";
      return false;
    }
    std::memcpy(d.params, &p, sizeof(p));
    use_nn<Attention>(d);
    d.family = "attention_bf16";
    d.flops = 4.0 * p.H * p.L * (double)p.L * p.dh;
    d.bytes = 2.0 * p.L * (3.0 * p.H * p.dh + p.H * p.dh);
    return true;
  }
  if (k == BL_OP_DWCONV) {
    DwParams p{};
    const int Nb = (int)op.dims[0];
    p.H = (int)op.dims[1]; p.Wd = (int)op.dims[2]; p.C = (int)op.dims[3];
    p.R_ = (int)op.dims[4]; p.S_ = (int)op.dims[5]; p.stride = (int)op.dims[6]; p.pad = (int)op.dims[7];
    p.X = (const bf16*)op.ptr[0]; p.W = (const bf16*)op.ptr[1];
    p.scale = (const float*)op.ptr[2]; p.shift = (const float*)op.ptr[3];
    p.R = (const bf16*)op.ptr[4]; p.Y = (bf16*)op.ptr[5];
    p.act = op.act;
    if (Nb != 1 || p.C % 8 || p.stride < 1 || !aligned16(p.X) || !aligned16(p.Y)) {
      err = "dwconv: batch 1, C % 8 == 0";
      return false;
    }
    p.OH = (p.H + 2 * p.pad - p.R_) / p.stride + 1;
    p.OW = (p.Wd + 2 * p.pad - p.S_) / p.stride + 1;
    p.items = (long long)p.OH * p.OW * (p.C / 8);
    long long per = (p.items + 2LL * caps.S - 1) / (2LL * caps.S);
    p.per_tile = (int)std::max<long long>(256, (per + 255) / 256 * 256);
    d.tiles = (uint32_t)((p.items + p.per_tile - 1) / p.per_tile);
    std::memcpy(d.params, &p, sizeof(p));
    use_nn<DwConv>(d);
    d.family = "dwconv_bf16";
    d.max_occ = 1;   // B200 sweep: fastest with 1 CTA/SM (profiles/round1/occ_cap.txt)
    d.flops = 2.0 * p.OH * p.OW * p.C * p.R_ * p.S_;
    d.bytes = 2.0 * ((double)p.H * p.Wd * p.C + (double)p.OH * p.OW * p.C * (p.R ? 2 : 1));
    return true;
  }
  // ELTWISE (bf16, strided)
  EwParams p{};
  p.X = (const bf16*)op.ptr[0];
  p.scale = (const float*)op.ptr[1];
  p.shift = (const float*)op.ptr[2];
  p.R = (const bf16*)op.ptr[3];
  p.Y = (bf16*)op.ptr[4];
  p.rows = (int)op.dims[0];
  p.C = (int)op.dims[1];
  p.ldx = op.dims[2] ? (int)op.dims[2] : p.C;
  p.ldy = op.dims[3] ? (int)op.dims[3] : p.C;
  p.act = op.act;
  if (p.C % 8 || p.ldx % 8 || p.ldy % 8 || !aligned16(p.X) || !aligned16(p.Y)) return false;  // generic path
  p.items = (long long)p.rows * (p.C / 8);
  long long per = (p.items + 2LL * caps.S - 1) / (2LL * caps.S);
  p.per_tile = (int)std::max<long long>(256, (per + 255) / 256 * 256);
  d.tiles = (uint32_t)((p.items + p.per_tile - 1) / p.per_tile);
  std::memcpy(d.params, &p, sizeof(p));
  use_nn<Eltwise>(d);
  d.family = "eltwise_bf16";
  d.max_occ = 1;   // B200 sweep: fastest with 1 CTA/SM (profiles/round1/occ_cap.txt)
  d.bytes = 2.0 * p.rows * p.C * (p.R ? 3 : 2);
  return true;
}

}  // namespace bless
