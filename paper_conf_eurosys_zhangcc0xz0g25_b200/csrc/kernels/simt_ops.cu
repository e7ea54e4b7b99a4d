// simt_ops.cu -- CUDA-core tenant kernels under the SM-gated executor.
//
//  * SimtMM: tiled fp32-accumulate GEMM / implicit-GEMM convolution (NHWC
//    input, KRSC weights) with the fused epilogue act(acc*scale+shift+R).
//    This is the fp32 path of config C1 (1e-4 parity) and
//    the generic fallback for shapes the tcgen05 path does not take.
//  * Pool: max / avg / global-average pooling, NHWC (K8).
//  * Eltwise: per-channel affine + activation (+ residual) (K7/K12).
//  * Gemv: M <= 8 rows (batch-1 FC layers): HBM-bound, 16-byte vector loads,
//    split over N rows and K chunks (K2 GEMV shapes).
// The tenants' layers come from the paper's applications (PAPER.md L259,
// L284); semantics as in oracle/layers_ref.py.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstring>

#include "../runtime/kdesc.hpp"
#include "executor.cuh"

namespace bless {

template <typename T>
__device__ __forceinline__ float ldf(const T* p);
template <>
__device__ __forceinline__ float ldf<float>(const float* p) { return __ldg(p); }
template <>
__device__ __forceinline__ float ldf<__nv_bfloat16>(const __nv_bfloat16* p) { return __bfloat162float(*p); }
__device__ __forceinline__ float to_f(float v) { return v; }
__device__ __forceinline__ float to_f(__nv_bfloat16 v) { return __bfloat162float(v); }
template <typename T>
__device__ __forceinline__ void stf(T* p, float v);
template <>
__device__ __forceinline__ void stf<float>(float* p, float v) { *p = v; }
template <>
__device__ __forceinline__ void stf<__nv_bfloat16>(__nv_bfloat16* p, float v) { *p = __float2bfloat16_rn(v); }

__device__ __forceinline__ float apply_act(float y, int act) {
  switch (act) {
    case BL_ACT_RELU: return fmaxf(y, 0.f);
    case BL_ACT_RELU6: return fminf(fmaxf(y, 0.f), 6.f);
    case BL_ACT_GELU: return 0.5f * y * (1.f + erff(y * 0.70710678118654752f));
    default: return y;
  }
}

// ---------------------------------------------------------------------------
// SimtMM
// ---------------------------------------------------------------------------
struct SimtMMParams {
  const void* X;
  const void* W;
  const float* scale;
  const float* shift;
  const void* R;
  void* Y;
  int M, N, K;
  int ldx, ldy, ldr;
  int act, conv;
  int H, Wd, C, OH, OW, R_, S_, stride, pad;
  int tiles_n;
};

constexpr int kMMB = 32;      // BM = BN = BK
constexpr int kMMThreads = 256;

template <typename T>
struct SimtMM {
  using Params = SimtMMParams;
  __device__ static float loadA(const Params& p, int m, int k) {
    const T* X = (const T*)p.X;
    if (!p.conv) return ldf(X + (size_t)m * p.ldx + k);
    const int hw = p.OH * p.OW;
    const int n = m / hw, pix = m - n * hw;
    const int oh = pix / p.OW, ow = pix - oh * p.OW;
    const int sc = p.S_ * p.C;
    const int r = k / sc, rem = k - r * sc;
    const int s = rem / p.C, c = rem - s * p.C;
    const int ih = oh * p.stride - p.pad + r, iw = ow * p.stride - p.pad + s;
    if (ih < 0 || ih >= p.H || iw < 0 || iw >= p.Wd) return 0.f;
    return ldf(X + ((size_t)(n * p.H + ih) * p.Wd + iw) * p.ldx + c);
  }
  __device__ static void tile(const Params& p, int t, unsigned char* smem) {
    float(*As)[kMMB + 1] = reinterpret_cast<float(*)[kMMB + 1]>(smem);
    float(*Bs)[kMMB + 1] = reinterpret_cast<float(*)[kMMB + 1]>(smem + sizeof(float) * kMMB * (kMMB + 1));
    const int tm = t / p.tiles_n, tn = t - tm * p.tiles_n;
    const int m0 = tm * kMMB, n0 = tn * kMMB;
    const int tid = threadIdx.x, ty = tid >> 4, tx = tid & 15;
    const T* W = (const T*)p.W;
    float acc[2][2] = {{0.f, 0.f}, {0.f, 0.f}};
    for (int k0 = 0; k0 < p.K; k0 += kMMB) {
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int idx = tid + i * kMMThreads;
        const int r = idx >> 5, c = idx & 31;
        const int m = m0 + r, n = n0 + r, k = k0 + c;
        As[c][r] = (m < p.M && k < p.K) ? loadA(p, m, k) : 0.f;
        Bs[c][r] = (n < p.N && k < p.K) ? ldf(W + (size_t)n * p.K + k) : 0.f;
      }
      __syncthreads();
#pragma unroll 8
      for (int kk = 0; kk < kMMB; ++kk) {
        const float a0 = As[kk][ty * 2], a1 = As[kk][ty * 2 + 1];
        const float b0 = Bs[kk][tx * 2], b1 = Bs[kk][tx * 2 + 1];
        acc[0][0] = fmaf(a0, b0, acc[0][0]);
        acc[0][1] = fmaf(a0, b1, acc[0][1]);
        acc[1][0] = fmaf(a1, b0, acc[1][0]);
        acc[1][1] = fmaf(a1, b1, acc[1][1]);
      }
      __syncthreads();
    }
    T* Y = (T*)p.Y;
    const T* Rr = (const T*)p.R;
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const int m = m0 + ty * 2 + i, n = n0 + tx * 2 + j;
        if (m >= p.M || n >= p.N) continue;
        float y = acc[i][j];
        if (p.scale) y *= __ldg(p.scale + n);
        if (p.shift) y += __ldg(p.shift + n);
        if (Rr) y += ldf(Rr + (size_t)m * p.ldr + n);
        stf(Y + (size_t)m * p.ldy + n, apply_act(y, p.act));
      }
  }
};

// ---------------------------------------------------------------------------
// Pool
// ---------------------------------------------------------------------------
struct PoolParams {
  const void* X;
  void* Y;
  int Nb, H, W, C, OH, OW, k, stride, pad, mode;
  int vec;              // elements per vector access (C % vec == 0)
  int ldy;              // output channel stride (window pools; DenseNet concat slices)
  long long items;      // output pixels x C/vec (window pools) | Nb x C/vec (global)
  int per_tile;         // items per tile (window pools) | vector groups per tile (global)
};

template <typename T>
struct VecT;  // 16-byte vector of T
template <>
struct VecT<__nv_bfloat16> {
  static constexpr int N = 8;
};
template <>
struct VecT<float> {
  static constexpr int N = 4;
};

template <typename T, int V>
__device__ __forceinline__ void load_vec(const T* p, float (&f)[V]) {
  if constexpr (V == 1) {
    f[0] = to_f(*p);
  } else {
    const uint4 u = __ldg(reinterpret_cast<const uint4*>(p));
    const T* e = reinterpret_cast<const T*>(&u);
#pragma unroll
    for (int i = 0; i < V; ++i) f[i] = to_f(e[i]);
  }
}
template <typename T, int V>
__device__ __forceinline__ void store_vec(T* p, const float (&f)[V]) {
  if constexpr (V == 1) {
    stf(p, f[0]);
  } else {
    uint4 u;
    T* e = reinterpret_cast<T*>(&u);
#pragma unroll
    for (int i = 0; i < V; ++i) {
      if constexpr (sizeof(T) == 2) e[i] = __float2bfloat16_rn(f[i]);
      else e[i] = f[i];
    }
    *reinterpret_cast<uint4*>(p) = u;
  }
}

// Window pools: one thread per (output pixel, vector of channels); the k*k
// window loads are independent 16-byte loads.  Global average: a tile is a
// block of channel vectors x all pixels, split over 8 pixel slices and
// reduced in shared memory.
template <typename T, int V>
struct Pool {
  using Params = PoolParams;
  __device__ static void tile(const Params& p, int t, unsigned char* smem) {
    const T* X = (const T*)p.X;
    T* Y = (T*)p.Y;
    const int CV = p.C / V;
    if (p.mode == BL_POOL_GLOBAL_AVG) {
      // per_tile vector groups; 256 threads = per_tile groups x (256/per_tile) slices
      const int gpt = p.per_tile, slices = blockDim.x / gpt;
      const int tiles_per_img = (CV + gpt - 1) / gpt;
      const int n = t / tiles_per_img, g0 = (t - n * tiles_per_img) * gpt;
      const int gl = threadIdx.x % gpt, sl = threadIdx.x / gpt;
      const int g = g0 + gl;
      const int hw = p.H * p.W;
      float acc[V];
#pragma unroll
      for (int i = 0; i < V; ++i) acc[i] = 0.f;
      if (g < CV) {
        const T* base = X + (size_t)n * hw * p.C + (size_t)g * V;
#pragma unroll 4
        for (int px = sl; px < hw; px += slices) {
          float f[V];
          load_vec<T, V>(base + (size_t)px * p.C, f);
#pragma unroll
          for (int i = 0; i < V; ++i) acc[i] += f[i];
        }
      }
      float* red = reinterpret_cast<float*>(smem);  // [slices][gpt][V]
      __syncthreads();
#pragma unroll
      for (int i = 0; i < V; ++i) red[(sl * gpt + gl) * V + i] = acc[i];
      __syncthreads();
      if (sl == 0 && g < CV) {
        for (int s2 = 1; s2 < slices; ++s2)
#pragma unroll
          for (int i = 0; i < V; ++i) acc[i] += red[(s2 * gpt + gl) * V + i];
#pragma unroll
        for (int i = 0; i < V; ++i) acc[i] /= (float)hw;
        store_vec<T, V>(Y + (size_t)n * p.C + (size_t)g * V, acc);
      }
      return;
    }
    const long long it0 = (long long)t * p.per_tile;
    const long long it1 = min(it0 + p.per_tile, p.items);
    for (long long it = it0 + threadIdx.x; it < it1; it += blockDim.x) {
      const int cv = (int)(it % CV);
      const long long pix = it / CV;
      const int n = (int)(pix / (p.OH * p.OW));
      const int q = (int)(pix - (long long)n * p.OH * p.OW);
      const int oh = q / p.OW, ow = q - oh * p.OW;
      float acc[V];
#pragma unroll
      for (int i = 0; i < V; ++i) acc[i] = (p.mode == BL_POOL_MAX) ? -INFINITY : 0.f;
      const int h0 = oh * p.stride - p.pad, w0 = ow * p.stride - p.pad;
      for (int r = 0; r < p.k; ++r) {
        const int ih = h0 + r;
        if (ih < 0 || ih >= p.H) continue;   // max: -inf padding; avg: zero padding (count_include_pad)
#pragma unroll 3
        for (int s = 0; s < p.k; ++s) {
          const int iw = w0 + s;
          if (iw < 0 || iw >= p.W) continue;
          float f[V];
          load_vec<T, V>(X + ((size_t)(n * p.H + ih) * p.W + iw) * p.C + (size_t)cv * V, f);
#pragma unroll
          for (int i = 0; i < V; ++i) acc[i] = (p.mode == BL_POOL_MAX) ? fmaxf(acc[i], f[i]) : acc[i] + f[i];
        }
      }
      if (p.mode == BL_POOL_AVG) {
#pragma unroll
        for (int i = 0; i < V; ++i) acc[i] /= (float)(p.k * p.k);
      }
      store_vec<T, V>(Y + (size_t)pix * p.ldy + (size_t)cv * V, acc);
    }
  }
};

// ---------------------------------------------------------------------------
// Im2col: Y[m, k] (row-major, Kpad columns) for a conv with few input channels,
// so that the conv itself runs as a tensor-core GEMM (first layers, C = 3).
// A tile is a run of `pw` output pixels of one output row.  The CTA first
// stages the R input rows x Wl columns x C channels it needs in shared memory
// (coalesced loads, padding zero-filled), then every thread assembles 16-byte
// output vectors from shared memory -- no per-element bounds checks or
// scattered global loads -- and consecutive threads store consecutive
// vectors.  (The former one-vector-per-thread gather from global memory ran at
// ~0.5 TB/s: VGG conv1 13.7 us, ResNet50 stem 10.1 us.)
// ---------------------------------------------------------------------------
struct Im2colParams {
  const void* X;
  void* Y;
  int H, W, C, R, S, stride, pad, Kpad, OH, OW;
  long long total;
  int pw, tiles_w, Wl;   // pixels per tile, tiles per output row, staged input width
};

template <typename T>
struct Im2col {
  using Params = Im2colParams;
  static constexpr int V = 16 / sizeof(T);   // one 16-byte output vector per thread step
  __device__ static void tile(const Params& p, int t, unsigned char* smem) {
    const T* X = (const T*)p.X;
    T* Y = (T*)p.Y;
    T* xs = reinterpret_cast<T*>(smem);      // [R][Wl][C]
    const int row = t / p.tiles_w, tw = t - row * p.tiles_w;
    const int n = row / p.OH, oh = row - n * p.OH;
    const int ow0 = tw * p.pw, np = min(p.pw, p.OW - ow0);
    const int h0 = oh * p.stride - p.pad, w0 = ow0 * p.stride - p.pad;
    const int WC = p.Wl * p.C, nst = p.R * WC;
    for (int i = threadIdx.x; i < nst; i += blockDim.x) {
      const int r = i / WC, rem = i - r * WC;
      const int x = rem / p.C, c = rem - x * p.C;
      const int ih = h0 + r, iw = w0 + x;
      T v = T(0.f);
      if (ih >= 0 && ih < p.H && iw >= 0 && iw < p.W) v = X[((size_t)(n * p.H + ih) * p.W + iw) * p.C + c];
      xs[i] = v;
    }
    __syncthreads();
    const int K = p.R * p.S * p.C;
    const int KV = p.Kpad / V;
    const int SC = p.S * p.C;
    const size_t m0 = (size_t)row * p.OW + ow0;
    for (int vi = threadIdx.x; vi < np * KV; vi += blockDim.x) {
      const int q = vi / KV;
      const int k0 = (vi - q * KV) * V;
      int r = k0 / SC;
      int rem = k0 - r * SC;                   // s * C + c within the tap row
      const int xq = q * p.stride * p.C;       // this pixel's window start in the staged row
      float f[V];
#pragma unroll
      for (int j = 0; j < V; ++j) {
        f[j] = (k0 + j < K) ? (float)xs[r * WC + xq + rem] : 0.f;
        if (++rem == SC) { rem = 0; ++r; }
      }
      store_vec<T, V>(Y + (m0 + q) * p.Kpad + k0, f);
    }
  }
};

// ---------------------------------------------------------------------------
// Eltwise: Y[r, c] = act(X*scale[c] + shift[c] + R)
// ---------------------------------------------------------------------------
struct EltParams {
  const void* X;
  const float* scale;
  const float* shift;
  const void* R;
  void* Y;
  long long total;
  int C, act, per_tile;
};

template <typename T>
struct Eltwise {
  using Params = EltParams;
  __device__ static void tile(const Params& p, int t, unsigned char*) {
    const long long e0 = (long long)t * p.per_tile;
    const long long e1 = min(e0 + p.per_tile, p.total);
    const T* X = (const T*)p.X;
    const T* R = (const T*)p.R;
    T* Y = (T*)p.Y;
    for (long long e = e0 + threadIdx.x; e < e1; e += blockDim.x) {
      const int c = (int)(e % p.C);
      float y = ldf(X + e);
      if (p.scale) y *= __ldg(p.scale + c);
      if (p.shift) y += __ldg(p.shift + c);
      if (R) y += ldf(R + e);
      stf(Y + e, apply_act(y, p.act));
    }
  }
};

// ---------------------------------------------------------------------------
// Gemv: Y[m, n] for m < M <= 8; tile = (row block of 8 outputs, K split).
// Each warp owns one output row n and streams W[n, k-chunk] with 16-byte
// loads; partial sums of a split-K tile are combined by atomics into an fp32
// workspace and the last split applies the epilogue (counter per row block).
// ---------------------------------------------------------------------------
struct GemvParams {
  const void* X;
  const void* W;
  const float* scale;
  const float* shift;
  const void* R;
  void* Y;
  int M, N, K, ldx, ldy, ldr, act;
  int rows_per_tile, ksplit, kchunk;
  float* ws;          // [M, N] fp32 partial sums (zeroed)
  unsigned* cnt;      // [row blocks] arrival counters (zeroed)
};

template <typename T>
struct Gemv {
  using Params = GemvParams;
  static constexpr int kVec = 16 / sizeof(T);
  __device__ static void tile(const Params& p, int t, unsigned char*) {
    const int rb = t / p.ksplit, ks = t - rb * p.ksplit;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nwarps = blockDim.x >> 5;
    const int k0 = ks * p.kchunk, k1 = min(p.K, k0 + p.kchunk);
    const T* X = (const T*)p.X;
    const T* W = (const T*)p.W;
    for (int rr = warp; rr < p.rows_per_tile; rr += nwarps) {
      const int n = rb * p.rows_per_tile + rr;
      if (n >= p.N) break;
      float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
      const T* wrow = W + (size_t)n * p.K;
      int k = k0 + lane * kVec;
      const bool vec_ok = ((p.K % kVec) == 0) && ((k0 % kVec) == 0) && ((p.ldx % kVec) == 0);
      if (vec_ok) {
        // kU independent 16-byte weight loads per lane in flight (memory-level
        // parallelism: a batch-1 FC layer is a pure weight stream from HBM)
        constexpr int kU = 8;
        constexpr int kStep = 32 * kVec;
        for (; k + (kU - 1) * kStep + kVec <= k1; k += kU * kStep) {
          uint4 wv[kU];
#pragma unroll
          for (int u = 0; u < kU; ++u)
            asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(wv[u].x), "=r"(wv[u].y), "=r"(wv[u].z), "=r"(wv[u].w)
                         : "l"(wrow + k + u * kStep));
#pragma unroll
          for (int u = 0; u < kU; ++u) {
            const T* we = reinterpret_cast<const T*>(&wv[u]);
            _Pragma("unroll") for (int m = 0; m < 8; ++m) if (m < p.M) {
              float xf[kVec];
              load_vec<T, kVec>(X + (size_t)m * p.ldx + k + u * kStep, xf);
              float s = 0.f;
#pragma unroll
              for (int v = 0; v < kVec; ++v) s = fmaf(to_f(we[v]), xf[v], s);
              acc[m] += s;
            }
          }
        }
        for (; k + kVec <= k1; k += kStep) {
          const uint4 wv = __ldg(reinterpret_cast<const uint4*>(wrow + k));
          const T* we = reinterpret_cast<const T*>(&wv);
          _Pragma("unroll") for (int m = 0; m < 8; ++m) if (m < p.M) {
            float xf[kVec];
            load_vec<T, kVec>(X + (size_t)m * p.ldx + k, xf);
            float s = 0.f;
#pragma unroll
            for (int v = 0; v < kVec; ++v) s = fmaf(to_f(we[v]), xf[v], s);
            acc[m] += s;
          }
        }
      } else {
        for (k = k0 + lane; k < k1; k += 32) {
          const float w = ldf(wrow + k);
          for (int m = 0; m < p.M && m < 8; ++m) acc[m] = fmaf(w, ldf(X + (size_t)m * p.ldx + k), acc[m]);
        }
      }
      _Pragma("unroll") for (int m = 0; m < 8; ++m) if (m < p.M) {
        float v = acc[m];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        acc[m] = v;
      }
      if (p.ksplit == 1) {
        if (lane == 0) {
          for (int m = 0; m < p.M; ++m) {
            float y = acc[m];
            if (p.scale) y *= __ldg(p.scale + n);
            if (p.shift) y += __ldg(p.shift + n);
            if (p.R) y += ldf((const T*)p.R + (size_t)m * p.ldr + n);
            stf((T*)p.Y + (size_t)m * p.ldy + n, apply_act(y, p.act));
          }
        }
      } else if (lane == 0) {
        for (int m = 0; m < p.M; ++m) atomicAdd(p.ws + (size_t)m * p.N + n, acc[m]);
      }
    }
    if (p.ksplit > 1) {
      __shared__ unsigned s_last;
      __syncthreads();
      if (threadIdx.x == 0) {
        __threadfence();
        s_last = (atomicAdd(p.cnt + rb, 1u) == (unsigned)p.ksplit - 1);
      }
      __syncthreads();
      if (s_last) {
        __threadfence();
        const int nb0 = rb * p.rows_per_tile;
        for (int i = threadIdx.x; i < p.rows_per_tile * p.M; i += blockDim.x) {
          const int rr = i % p.rows_per_tile, m = i / p.rows_per_tile;
          const int n = nb0 + rr;
          if (n >= p.N) continue;
          volatile float* wsv = p.ws + (size_t)m * p.N + n;
          float y = *wsv;
          *wsv = 0.f;  // leave the workspace zeroed for the next launch
          if (p.scale) y *= __ldg(p.scale + n);
          if (p.shift) y += __ldg(p.shift + n);
          if (p.R) y += ldf((const T*)p.R + (size_t)m * p.ldr + n);
          stf((T*)p.Y + (size_t)m * p.ldy + n, apply_act(y, p.act));
        }
        if (threadIdx.x == 0) p.cnt[rb] = 0;
      }
    }
  }
};

// ---------------------------------------------------------------------------
// gated kernels + launchers
// ---------------------------------------------------------------------------
template <class Op>
__global__ void __launch_bounds__(256) k_gated(const typename Op::Params p, const GateArgs g) {
  extern __shared__ __align__(16) unsigned char smem[];
  gated_run<Op>(p, g, smem);
}

template <class Op>
static cudaError_t launch_gated(const KernelDesc& d, const GateArgs& g, cudaStream_t st) {
  void* args[2] = {(void*)d.params, (void*)&g};
  return launch_kernel((const void*)k_gated<Op>, dim3(launch_grid(d, g)), dim3(d.block), (size_t)d.smem, st, args);
}

template <class Op>
static void use_gated(KernelDesc& d) {
  d.launch = launch_gated<Op>;
  d.kernel_fn = (const void*)k_gated<Op>;
}

static inline size_t esize(int dt) { return dt == BL_BF16 ? 2 : 4; }

// Gemv split-K workspace: one static pool per process (zero-initialised, each
// launch leaves it zeroed).  Kernels of the same tenant never run
// concurrently (one stream), but different tenants may: give every Gemv
// kernel its own region.
static float* gemv_ws_alloc(size_t floats, size_t counters, unsigned** cnt_out) {
  void* p = nullptr;
  if (cudaMalloc(&p, floats * 4 + counters * 4) != cudaSuccess) return nullptr;
  cudaMemset(p, 0, floats * 4 + counters * 4);
  *cnt_out = reinterpret_cast<unsigned*>(reinterpret_cast<char*>(p) + floats * 4);
  return reinterpret_cast<float*>(p);
}

bool build_simt(const bl_op& op, const DeviceCaps& caps, KernelDesc& d, std::string& err) {
  const bool bf = op.dtype == BL_BF16;
  if (op.dtype != BL_F32 && op.dtype != BL_BF16) { err = "dtype"; return false; }
  const int occ = 2;
  d.block = 256;
  d.grid = caps.S * occ;
  d.op = op;
  if (op.kind == BL_OP_GEMM || op.kind == BL_OP_CONV) {
    SimtMMParams p{};
    p.X = op.ptr[0]; p.W = op.ptr[1]; p.scale = (const float*)op.ptr[2]; p.shift = (const float*)op.ptr[3];
    p.R = op.ptr[4]; p.Y = op.ptr[5]; p.act = op.act;
    if (op.kind == BL_OP_GEMM) {
      p.M = (int)op.dims[0]; p.N = (int)op.dims[1]; p.K = (int)op.dims[2];
      p.ldx = op.dims[3] ? (int)op.dims[3] : p.K;
      p.ldy = op.dims[4] ? (int)op.dims[4] : p.N;
      p.ldr = op.dims[5] ? (int)op.dims[5] : p.N;
      p.conv = 0;
      if (p.M <= 8 && p.M >= 1) {
        // batch-1 FC layer: HBM-bound GEMV path
        GemvParams q{};
        q.X = p.X; q.W = p.W; q.scale = p.scale; q.shift = p.shift; q.R = p.R; q.Y = p.Y;
        q.M = p.M; q.N = p.N; q.K = p.K; q.ldx = p.ldx; q.ldy = p.ldy; q.ldr = p.ldr; q.act = p.act;
        q.rows_per_tile = 8;
        const int rblocks = (q.N + 7) / 8;
        // split K so there are >= ~2 tiles per SM when K is long
        int ks = 1;
        while ((long long)rblocks * ks < 2LL * caps.S && q.K / (ks * 2) >= 1024) ks *= 2;
        q.ksplit = ks;
        const int vec = bf ? 8 : 4;
        q.kchunk = ((q.K + ks - 1) / ks + vec - 1) / vec * vec;
        if (ks > 1) {
          q.ws = gemv_ws_alloc((size_t)q.M * q.N, rblocks, &q.cnt);
          if (!q.ws) { err = "gemv workspace alloc"; return false; }
        }
        d.tiles = (uint32_t)(rblocks * ks);
        d.smem = 0;
        std::memcpy(d.params, &q, sizeof(q));
        if (bf) use_gated<Gemv<__nv_bfloat16>>(d);
        else use_gated<Gemv<float>>(d);
        d.family = bf ? "gemv_bf16" : "gemv_f32";
        d.flops = 2.0 * q.M * q.N * q.K;
        d.bytes = esize(op.dtype) * ((double)q.N * q.K + (double)q.M * q.K + (double)q.M * q.N);
        return true;
      }
    } else {
      const int Nb = (int)op.dims[0], H = (int)op.dims[1], Wd = (int)op.dims[2], C = (int)op.dims[3];
      const int K = (int)op.dims[4], R = (int)op.dims[5], S = (int)op.dims[6];
      const int stride = (int)op.dims[7], pad = (int)op.dims[8], groups = (int)op.dims[9];
      if (groups != 1) { err = "simt conv supports groups == 1 only"; return false; }
      if (stride < 1 || R < 1 || S < 1 || C < 1 || K < 1 || Nb < 1) { err = "conv dims"; return false; }
      p.H = H; p.Wd = Wd; p.C = C; p.R_ = R; p.S_ = S; p.stride = stride; p.pad = pad;
      p.OH = (H + 2 * pad - R) / stride + 1;
      p.OW = (Wd + 2 * pad - S) / stride + 1;
      p.M = Nb * p.OH * p.OW; p.N = K; p.K = R * S * C;
      p.ldx = op.dims[10] ? (int)op.dims[10] : C;
      p.ldy = op.dims[11] ? (int)op.dims[11] : K;
      p.ldr = p.ldy;
      p.conv = 1;
    }
    if (p.M < 0 || p.N < 1 || p.K < 1) { err = "gemm dims"; return false; }
    p.tiles_n = (p.N + kMMB - 1) / kMMB;
    d.tiles = (uint32_t)(((p.M + kMMB - 1) / kMMB) * p.tiles_n);
    d.smem = 2 * sizeof(float) * kMMB * (kMMB + 1);
    std::memcpy(d.params, &p, sizeof(p));
    if (bf) use_gated<SimtMM<__nv_bfloat16>>(d);
    else use_gated<SimtMM<float>>(d);
    d.family = bf ? "simt_mm_bf16" : "simt_mm_f32";
    d.flops = 2.0 * p.M * p.N * p.K;
    d.bytes = esize(op.dtype) * ((double)p.N * p.K + (double)p.M * p.N * (p.R ? 2 : 1) +
                                 (op.kind == BL_OP_CONV ? (double)op.dims[0] * op.dims[1] * op.dims[2] * op.dims[3]
                                                        : (double)p.M * p.K));
    return true;
  }
  if (op.kind == BL_OP_POOL) {
    PoolParams p{};
    p.X = op.ptr[0]; p.Y = op.ptr[1];
    p.Nb = (int)op.dims[0]; p.H = (int)op.dims[1]; p.W = (int)op.dims[2]; p.C = (int)op.dims[3];
    p.k = (int)op.dims[4]; p.stride = (int)op.dims[5]; p.pad = (int)op.dims[6]; p.mode = (int)op.dims[7];
    p.ldy = op.dims[8] ? (int)op.dims[8] : p.C;
    if (p.C < 1 || p.Nb < 1) { err = "pool dims"; return false; }
    const int V = bf ? 8 : 4;
    const bool vec = (p.C % V) == 0 && (p.ldy % V) == 0 && (((uintptr_t)p.X | (uintptr_t)p.Y) & 15) == 0;
    p.vec = vec ? V : 1;
    const int CV = p.C / p.vec;
    if (p.mode == BL_POOL_GLOBAL_AVG) {
      p.OH = p.OW = 1;
      p.per_tile = 16;                       // vector groups per tile (x 16 pixel slices)
      d.tiles = (uint32_t)(p.Nb * ((CV + p.per_tile - 1) / p.per_tile));
      d.smem = 256 * 8 * sizeof(float);
    } else {
      if (p.k < 1 || p.stride < 1) { err = "pool dims"; return false; }
      p.OH = (p.H + 2 * p.pad - p.k) / p.stride + 1;
      p.OW = (p.W + 2 * p.pad - p.k) / p.stride + 1;
      p.items = (long long)p.Nb * p.OH * p.OW * CV;
      // ~2 tiles per SM, one item per thread per pass, at least 256 items
      long long per = (p.items + 2LL * caps.S - 1) / (2LL * caps.S);
      per = std::max<long long>(256, (per + 255) / 256 * 256);
      p.per_tile = (int)std::min<long long>(per, 1 << 16);
      d.tiles = (uint32_t)((p.items + p.per_tile - 1) / p.per_tile);
      d.smem = 0;
    }
    std::memcpy(d.params, &p, sizeof(p));
    if (bf && vec) use_gated<Pool<__nv_bfloat16, 8>>(d);
    else if (bf) use_gated<Pool<__nv_bfloat16, 1>>(d);
    else if (vec) use_gated<Pool<float, 4>>(d);
    else use_gated<Pool<float, 1>>(d);
    d.family = bf ? "pool_bf16" : "pool_f32";
    d.max_occ = 2;   // B200 sweep (profiles/round1/occ_cap.txt)
    d.bytes = esize(op.dtype) * ((double)p.Nb * p.H * p.W * p.C + (double)p.Nb * p.OH * p.OW * p.C);
    return true;
  }
  if (op.kind == BL_OP_IM2COL) {
    Im2colParams p{};
    p.X = op.ptr[0];
    p.Y = op.ptr[1];
    const int Nb = (int)op.dims[0];
    p.H = (int)op.dims[1]; p.W = (int)op.dims[2]; p.C = (int)op.dims[3];
    p.R = (int)op.dims[4]; p.S = (int)op.dims[5]; p.stride = (int)op.dims[6]; p.pad = (int)op.dims[7];
    p.Kpad = (int)op.dims[8];
    if (Nb < 1 || p.C < 1 || p.R < 1 || p.S < 1 || p.stride < 1 || p.Kpad < p.R * p.S * p.C) {
      err = "im2col dims";
      return false;
    }
    p.OH = (p.H + 2 * p.pad - p.R) / p.stride + 1;
    p.OW = (p.W + 2 * p.pad - p.S) / p.stride + 1;
    p.total = (long long)Nb * p.OH * p.OW * p.Kpad;
    const int V = bf ? 8 : 4;
    if (p.Kpad % V || (((uintptr_t)p.Y) & 15) || p.total / V >= (1LL << 31)) { err = "im2col: Kpad/alignment"; return false; }
    // tile = pw output pixels of one row: about 3 tiles per SM, staged input <= 32 KB
    const long long rows = (long long)Nb * p.OH;
    int split = (int)std::max<long long>(1, (3LL * caps.S + rows - 1) / rows);
    split = std::min(split, p.OW);
    p.pw = (p.OW + split - 1) / split;
    auto staged = [&](int pw) { return (long long)p.R * ((pw - 1) * p.stride + p.S) * p.C * (bf ? 2 : 4); };
    while (p.pw > 1 && staged(p.pw) > 32768) p.pw = (p.pw + 1) / 2;
    p.tiles_w = (p.OW + p.pw - 1) / p.pw;
    p.Wl = (p.pw - 1) * p.stride + p.S;
    d.tiles = (uint32_t)(rows * p.tiles_w);
    d.smem = (int)((staged(p.pw) + 15) / 16 * 16);
    std::memcpy(d.params, &p, sizeof(p));
    if (bf) use_gated<Im2col<__nv_bfloat16>>(d);
    else use_gated<Im2col<float>>(d);
    d.family = bf ? "im2col_bf16" : "im2col_f32";
    d.max_occ = 4;   // B200 sweep (profiles/round1/occ_cap.txt)
    d.bytes = esize(op.dtype) * ((double)Nb * p.H * p.W * p.C + (double)p.total);
    return true;
  }
  if (op.kind == BL_OP_ELTWISE) {
    EltParams p{};
    p.X = op.ptr[0]; p.scale = (const float*)op.ptr[1]; p.shift = (const float*)op.ptr[2]; p.R = op.ptr[3];
    p.Y = op.ptr[4];
    p.total = op.dims[0] * op.dims[1];
    p.C = (int)op.dims[1];
    p.act = op.act;
    p.per_tile = 8192;
    if (p.C < 1) { err = "eltwise dims"; return false; }
    d.tiles = (uint32_t)((p.total + p.per_tile - 1) / p.per_tile);
    d.smem = 0;
    std::memcpy(d.params, &p, sizeof(p));
    if (bf) use_gated<Eltwise<__nv_bfloat16>>(d);
    else use_gated<Eltwise<float>>(d);
    d.family = bf ? "eltwise_bf16" : "eltwise_f32";
    d.max_occ = 1;   // B200 sweep (profiles/round1/occ_cap.txt)
    d.bytes = esize(op.dtype) * (double)p.total * (p.R ? 3 : 2);
    return true;
  }
  err = "unsupported op kind";
  return false;
}

}  // namespace bless
