// tma_bench.cu -- per-SM TMA load throughput on B200 for the box shapes the
// tcgen05 GEMM/conv kernels use (cost model of the operand feed).
//
// One CTA per SM, one thread issues TMA loads of a given box into a ring of
// ST shared-memory stages (no consumer work: a stage is re-armed as soon as its
// previous load has landed), N boxes per CTA, coordinates walking over an
// L2-resident tensor.  Reports ns per box and bytes per SM clock.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_bench tools/tma_bench.cu -lcuda && ./tma_bench
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <string>
#include <vector>

struct __align__(64) Maps {
  CUtensorMap m;
};

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int RANK>
__global__ void k_tma(const __grid_constant__ Maps mp, int ST, int nbox, int box_bytes, int d1, int d2, int d3,
                      int m1, int m2, int m3, unsigned long long* out) {
  extern __shared__ __align__(1024) unsigned char sm_raw[];
  unsigned char* sm = (unsigned char*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar[16];
  if (threadIdx.x != 0) return;
  for (int i = 0; i < ST; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[i])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  asm volatile("prefetch.tensormap [%0];" ::"l"(&mp.m) : "memory");
  unsigned long long t0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  uint32_t ph[16] = {0};
  for (int i = 0; i < nbox; ++i) {
    const int s = i % ST;
    if (i >= ST) {
      asm volatile(
          "{\n\t.reg .pred p;\n\tW_%=:\n\t"
          "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n\t}" ::"r"(su32(&bar[s])),
          "r"(ph[s])
          : "memory");
      ph[s] ^= 1;
    }
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(box_bytes)
                 : "memory");
    const int c1 = ((blockIdx.x * 7 + i) % d1) * m1, c2 = ((blockIdx.x * 3 + i / d1) % d2) * m2,
              c3 = ((i / (d1 * d2)) % d3) * m3;
    void* dst = sm + (size_t)s * box_bytes;
    if (RANK == 2)
      asm volatile(
          "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
          ::"r"(su32(dst)), "l"(&mp.m), "r"(su32(&bar[s])), "r"(0), "r"(c1) : "memory");
    else if (RANK == 3)
      asm volatile(
          "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], "
          "[%2];" ::"r"(su32(dst)), "l"(&mp.m), "r"(su32(&bar[s])), "r"(0), "r"(c1), "r"(c2) : "memory");
    else
      asm volatile(
          "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], "
          "[%2];" ::"r"(su32(dst)), "l"(&mp.m), "r"(su32(&bar[s])), "r"(0), "r"(c1 - 1), "r"(c2 - 1), "r"(c3)
          : "memory");
  }
  for (int i = nbox; i < nbox + ST; ++i) {
    const int s = i % ST;
    if (i >= ST) {
      asm volatile(
          "{\n\t.reg .pred p;\n\tW_%=:\n\t"
          "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n\t}" ::"r"(su32(&bar[s])),
          "r"(ph[s])
          : "memory");
      ph[s] ^= 1;
    }
  }
  unsigned long long t1;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
  out[blockIdx.x] = t1 - t0;
}

// Same ring with the engine's handoff: warp 0 (one thread) issues loads into
// stage s after waiting on empty[s]; warp 1 waits on full[s] and arrives on
// empty[s] (what the MMA warp does after its MMAs).  Measures the cost of the
// two mbarrier handoffs per stage on top of the TMA time.
template <int RANK>
__global__ void k_tma_pc(const __grid_constant__ Maps mp, int ST, int nbox, int box_bytes, int d1, int d2, int d3,
                         int m1, int m2, int m3, unsigned long long* out) {
  extern __shared__ __align__(1024) unsigned char sm_raw[];
  unsigned char* sm = (unsigned char*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t full[16], empty[16];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < ST; ++i) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[i])));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&empty[i])));
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  unsigned long long t0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  if (warp == 0 && lane == 0) {
    for (int i = 0; i < nbox; ++i) {
      const int s = i % ST;
      const uint32_t ph = ((i / ST) & 1) ^ 1;
      asm volatile(
          "{\n\t.reg .pred p;\n\tW_%=:\n\t"
          "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n\t}" ::"r"(su32(&empty[s])),
          "r"(ph)
          : "memory");
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(box_bytes)
                   : "memory");
      const int c1 = ((blockIdx.x * 7 + i) % d1) * m1, c2 = ((blockIdx.x * 3 + i / d1) % d2) * m2,
                c3 = ((i / (d1 * d2)) % d3) * m3;
      void* dst = sm + (size_t)s * box_bytes;
      if (RANK == 2)
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
            ::"r"(su32(dst)), "l"(&mp.m), "r"(su32(&full[s])), "r"(0), "r"(c1) : "memory");
      else
        asm volatile(
            "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], "
            "[%2];" ::"r"(su32(dst)), "l"(&mp.m), "r"(su32(&full[s])), "r"(0), "r"(c1 - 1), "r"(c2 - 1), "r"(c3)
            : "memory");
    }
  } else if (warp == 1) {
    for (int i = 0; i < nbox; ++i) {
      const int s = i % ST;
      const uint32_t ph = (i / ST) & 1;
      asm volatile(
          "{\n\t.reg .pred p;\n\tW_%=:\n\t"
          "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n\t}" ::"r"(su32(&full[s])),
          "r"(ph)
          : "memory");
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[s])) : "memory");
      __syncwarp();
    }
    unsigned long long t1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
    if (lane == 0) out[blockIdx.x] = t1 - t0;
  }
}

// tcgen05.mma issue rate: one warp issues n MMAs (M = 128, N = BN, K = 16,
// bf16, A/B from zeroed shared memory, D in TMEM) and waits for their commit;
// 'elect' = warp-uniform loop with elect.sync, else `if (lane == 0)`.
// pattern 0: one 128 x 64 A tile and one BN x 64 B tile, K steps cycled;
// pattern 1: the halo conv's access pattern -- tap (r, s) reads A from a
// 58-pixel-wide halo at row offset r*58 + s (not 8-row aligned), B from a
// 3-tap weight stage; fill: 0 = zeros, 1 = bf16 ones.
template <int BN>
__global__ void k_mma_rate(int n, int elect, unsigned long long* out, int pattern = 0, int fill = 0, int accs = 1) {
  extern __shared__ __align__(1024) unsigned char sm_raw[];
  unsigned char* sm = (unsigned char*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar;
  __shared__ uint32_t tslot;
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < (256 + 3 * BN) * 128 / 4; i += 32) ((uint32_t*)sm)[i] = fill ? 0x3F803F80u : 0u;
  if (lane == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(su32(&tslot)));
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncwarp();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tm = __shfl_sync(0xffffffffu, tslot, 0);
  const uint32_t a = su32(sm), b = su32(sm + 256 * 128);
  auto desc = [](uint32_t addr) {
    uint64_t d = (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
                 ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
    return d;
  };
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
  unsigned long long t0, t1;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  if (elect) {
    for (int i = 0; i < n; ++i) {
      const uint32_t k = (i & 3) * 32;
      uint32_t ao = k, bo = k;
      if (pattern == 1) {
        const int tap = (i >> 2) % 9, r = tap / 3, s_ = tap - 3 * r;
        ao += (uint32_t)(r * 58 + s_) * 128u;
        bo += (uint32_t)s_ * (BN * 128u);
      }
      // accs > 1: consecutive MMAs rotate over independent TMEM accumulators
      const int acc = accs > 1 ? i % accs : 0;
      asm volatile(
          "{\n\t.reg .pred p, e;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
          "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tm + (uint32_t)(acc * BN)),
          "l"(desc(a + ao)), "l"(desc(b + bo)), "r"(idesc), "r"(i >= accs ? 1 : 0)
          : "memory");
    }
    asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
                 "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar))
                 : "memory");
  } else if (lane == 0) {
    for (int i = 0; i < n; ++i) {
      const uint32_t k = (i & 3) * 32;
      asm volatile(
          "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
          "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tm),
          "l"(desc(a + k)), "l"(desc(b + k)), "r"(idesc), "r"(i)
          : "memory");
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar))
                 : "memory");
  }
  asm volatile(
      "{\n\t.reg .pred p;\n\tW_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n\t@!p bra W_%=;\n\t}" ::"r"(su32(&bar))
      : "memory");
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
  if (lane == 0) out[blockIdx.x] = t1 - t0;
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncwarp();
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tm));
}

// MMAs under concurrent TMA traffic: warp 1 issues n MMAs (halo pattern, M =
// 128, N = BN) reading operands from smem [0, 64 KB); warp 0 meanwhile keeps
// ST 16 KB 2-D TMA boxes in flight into [96 KB, 96 KB + ST*16 KB) (tma = 1)
// or idles (tma = 0).  out[b] = MMA time, out[S + b] = boxes landed meanwhile.
template <int BN>
__global__ void k_mma_tma(const __grid_constant__ Maps mp, int n, int tma, int ST, unsigned long long* out) {
  extern __shared__ __align__(1024) unsigned char sm_raw[];
  unsigned char* sm = (unsigned char*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar, tb[8];
  __shared__ uint32_t tslot;
  __shared__ volatile int done;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) ((uint32_t*)sm)[i] = 0x3F803F80u;
  if (threadIdx.x == 0) {
    done = 0;
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    for (int i = 0; i < ST; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&tb[i])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(su32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (warp == 0) {
    if (lane != 0 || !tma) return;
    uint32_t ph[8] = {0};
    unsigned long long boxes = 0;
    for (int i = 0;; ++i) {
      const int s = i % ST;
      if (i >= ST) {
        asm volatile("{\n\t.reg .pred p;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
                     "@!p bra W_%=;\n\t}" ::"r"(su32(&tb[s])), "r"(ph[s]) : "memory");
        ph[s] ^= 1;
        ++boxes;
      }
      if (done) {
        for (int j = i + 1; j < i + ST; ++j) {   // drain the other in-flight stages
          const int s2 = j % ST;
          if (j >= ST) {
            asm volatile("{\n\t.reg .pred p;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
                         "@!p bra W_%=;\n\t}" ::"r"(su32(&tb[s2])), "r"(ph[s2]) : "memory");
            ph[s2] ^= 1;
          }
        }
        break;
      }
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&tb[s])), "r"(16384) : "memory");
      void* dst = sm + 96 * 1024 + (size_t)s * 16384;
      asm volatile(
          "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
          ::"r"(su32(dst)), "l"(&mp.m), "r"(su32(&tb[s])), "r"(0), "r"(((blockIdx.x * 7 + i) % 64) * 128) : "memory");
    }
    out[gridDim.x + blockIdx.x] = boxes;
    return;
  }
  if (warp != 1) return;
  const uint32_t tm = __shfl_sync(0xffffffffu, tslot, 0);
  const uint32_t a = su32(sm), b = su32(sm + 256 * 128);
  auto desc = [](uint32_t addr) {
    return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
           ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
  };
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
  unsigned long long t0, t1;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (int i = 0; i < n; ++i) {
    const int tap = (i >> 2) % 9, r = tap / 3, s_ = tap - 3 * r;
    const uint32_t ao = (i & 3) * 32 + (uint32_t)(r * 58 + s_) * 128u, bo = (i & 3) * 32 + (uint32_t)s_ * (BN * 128u);
    asm volatile(
        "{\n\t.reg .pred p, e;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tm),
        "l"(desc(a + ao)), "l"(desc(b + bo)), "r"(idesc), "r"(i)
        : "memory");
  }
  asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
               "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(su32(&bar))
               : "memory");
  asm volatile("{\n\t.reg .pred p;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n\t"
               "@!p bra W_%=;\n\t}" ::"r"(su32(&bar)) : "memory");
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
  if (lane == 0) {
    out[blockIdx.x] = t1 - t0;
    done = 1;
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncwarp();
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tm));
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main(int argc, char** argv) {
  const bool only_accs = argc > 1 && std::string(argv[1]) == "accs";
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  Enc enc = (Enc)fn;
  int S = 0;
  cudaDeviceGetAttribute(&S, cudaDevAttrMultiProcessorCount, 0);
  int clk_khz = 0;
  cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
  // NHWC 56 x 64 x 512 bf16 (3.7 MB) and a [8192, 512] matrix: L2 resident
  const int H = 56, W = 64, C = 512;
  void* X = nullptr;
  cudaMalloc(&X, (size_t)64 << 20);
  cudaMemset(X, 0, (size_t)64 << 20);
  unsigned long long* d_out;
  cudaMalloc(&d_out, S * sizeof(unsigned long long));
  std::vector<unsigned long long> h(S);
  struct Case {
    const char* name;
    int rank;
    cuuint64_t dims[4];
    cuuint64_t strides[3];
    cuuint32_t box[4];
    int d1, d2, d3;
  };
  std::vector<Case> cases = {
      {"2D (64ch, 64 rows) 8KB", 2, {64, 8192}, {(cuuint64_t)C * 2}, {64, 64}, 8192 / 64, 1, 1},
      {"2D (64ch, 128 rows) 16KB", 2, {64, 8192}, {(cuuint64_t)C * 2}, {64, 128}, 8192 / 128, 1, 1},
      {"2D (64ch, 256 rows) 32KB", 2, {64, 8192}, {(cuuint64_t)C * 2}, {64, 256}, 8192 / 256, 1, 1},
      {"3D (64, 128 rows, 2 slabs) 32KB", 3, {64, 8192, 8}, {(cuuint64_t)C * 2, 128}, {64, 128, 2}, 8192 / 128, 4, 1},
      {"3D (64, 64 rows, 2 slabs) 16KB", 3, {64, 8192, 8}, {(cuuint64_t)C * 2, 128}, {64, 64, 2}, 8192 / 64, 4, 1},
      {"4D conv (64ch, 64w, 2h, 1) 16KB", 4, {64, (cuuint64_t)W, (cuuint64_t)H, 8},
       {(cuuint64_t)C * 2, (cuuint64_t)W * C * 2, 128}, {64, 64, 2, 1}, 1, H / 2, 8},
      {"4D conv (64ch, 64w, 2h, 2 slabs) 32KB", 4, {64, (cuuint64_t)W, (cuuint64_t)H, 8},
       {(cuuint64_t)C * 2, (cuuint64_t)W * C * 2, 128}, {64, 64, 2, 2}, 1, H / 2, 4},
      {"4D halo (64ch, 64w, 4h, 1) 32KB", 4, {64, (cuuint64_t)W, (cuuint64_t)H, 8},
       {(cuuint64_t)C * 2, (cuuint64_t)W * C * 2, 128}, {64, 64, 4, 1}, 1, H / 4, 8},
      {"4D conv (16ch, 64w, 2h, 1) 4KB", 4, {64, (cuuint64_t)W, (cuuint64_t)H, 8},
       {(cuuint64_t)C * 2, (cuuint64_t)W * C * 2, 128}, {16, 64, 2, 1}, 1, H / 2, 8},
  };
  printf("S=%d sm_clock=%d MHz\n", S, clk_khz / 1000);
  {  // MMA rate vs independent accumulators (is the ~60-cycle floor of N <= 64 a dependency chain?)
    for (int bn : {32, 64, 128}) {
      const void* kf = bn == 32 ? (const void*)k_mma_rate<32>
                                : (bn == 64 ? (const void*)k_mma_rate<64> : (const void*)k_mma_rate<128>);
      cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
      for (int accs : {1, 2, 4}) {
        if (accs * bn > 256) continue;
        const int n = 2048;
        for (int rep = 0; rep < 2; ++rep) {
          if (bn == 32) k_mma_rate<32><<<S, 32, 160 * 1024>>>(n, 1, d_out, 0, 0, accs);
          else if (bn == 64) k_mma_rate<64><<<S, 32, 160 * 1024>>>(n, 1, d_out, 0, 0, accs);
          else k_mma_rate<128><<<S, 32, 160 * 1024>>>(n, 1, d_out, 0, 0, accs);
        }
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("mma: %s\n", cudaGetErrorString(e)); return 1; }
        cudaMemcpy(h.data(), d_out, S * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < S; ++i) avg += (double)h[i] / S;
        printf("MMA 128x%dx16 over %d accumulator(s): %.1f ns/mma = %.1f cycles (floor %d)\n", bn, accs, avg / n,
               avg / n * clk_khz / 1e6, 128 * bn / 256);
      }
    }
  }
  if (only_accs) return 0;
  // MMA issue rate
  for (int elect = 0; elect < 2; ++elect) {
    for (int bn : {64, 128, 256}) {
      const void* kf = bn == 64 ? (const void*)k_mma_rate<64> : (bn == 128 ? (const void*)k_mma_rate<128>
                                                                           : (const void*)k_mma_rate<256>);
      cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
      const int n = 2048;
      for (int rep = 0; rep < 2; ++rep) {
        if (bn == 64) k_mma_rate<64><<<S, 32, 160 * 1024>>>(n, elect, d_out);
        else if (bn == 128) k_mma_rate<128><<<S, 32, 160 * 1024>>>(n, elect, d_out);
        else k_mma_rate<256><<<S, 32, 160 * 1024>>>(n, elect, d_out);
      }
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("mma: %s\n", cudaGetErrorString(e)); return 1; }
      cudaMemcpy(h.data(), d_out, S * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
      double avg = 0;
      for (int i = 0; i < S; ++i) avg += (double)h[i] / S;
      const double cyc = avg / n * clk_khz / 1e6;
      printf("MMA 128x%dx16 %s: %.1f ns/mma = %.1f cycles (floor %d)  -> %.0f TF/s chip\n", bn,
             elect ? "elect.sync uniform loop" : "if (lane == 0)      ", avg / n, cyc, 128 * bn / 256,
             2.0 * 128 * bn * 16 / (avg / n) * S / 1e3);
    }
  }
  // halo access pattern and operand values (elect loop)
  for (int pattern = 0; pattern < 2; ++pattern)
    for (int fill = 0; fill < 2; ++fill)
      for (int bn : {32, 64, 128}) {
        const void* kf = bn == 32 ? (const void*)k_mma_rate<32>
                                  : (bn == 64 ? (const void*)k_mma_rate<64> : (const void*)k_mma_rate<128>);
        cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
        const int n = 2304;
        for (int rep = 0; rep < 2; ++rep) {
          if (bn == 32) k_mma_rate<32><<<S, 32, 160 * 1024>>>(n, 1, d_out, pattern, fill);
          else if (bn == 64) k_mma_rate<64><<<S, 32, 160 * 1024>>>(n, 1, d_out, pattern, fill);
          else k_mma_rate<128><<<S, 32, 160 * 1024>>>(n, 1, d_out, pattern, fill);
        }
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("mma: %s\n", cudaGetErrorString(e)); return 1; }
        cudaMemcpy(h.data(), d_out, S * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < S; ++i) avg += (double)h[i] / S;
        printf("MMA 128x%dx16 %s %s: %.1f ns/mma = %.1f cycles (floor %d)\n", bn,
               pattern ? "halo-offset A (r*58+s rows), 3-tap B" : "aligned A/B                       ",
               fill ? "ones " : "zeros", avg / n, avg / n * clk_khz / 1e6, 128 * bn / 256);
      }
  {  // MMAs under concurrent TMA traffic
    Maps mp;
    cuuint64_t dims[2] = {64, 8192}, strides[1] = {(cuuint64_t)C * 2};
    cuuint32_t box[2] = {64, 128}, es[2] = {1, 1};
    enc(&mp.m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, X, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    std::vector<unsigned long long> h2(2 * S);
    unsigned long long* d2;
    cudaMalloc(&d2, 2 * S * sizeof(unsigned long long));
    for (int bn : {64, 128})
      for (int tma = 0; tma < 2; ++tma)
        for (int ST : {2, 4}) {
          if (!tma && ST == 4) continue;
          const void* kf = bn == 64 ? (const void*)k_mma_tma<64> : (const void*)k_mma_tma<128>;
          cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
          const int n = 2304;
          cudaMemset(d2, 0, 2 * S * sizeof(unsigned long long));
          for (int rep = 0; rep < 2; ++rep) {
            if (bn == 64) k_mma_tma<64><<<S, 64, 196 * 1024>>>(mp, n, tma, ST, d2);
            else k_mma_tma<128><<<S, 64, 196 * 1024>>>(mp, n, tma, ST, d2);
          }
          cudaError_t e = cudaDeviceSynchronize();
          if (e != cudaSuccess) { printf("mma_tma: %s\n", cudaGetErrorString(e)); return 1; }
          cudaMemcpy(h2.data(), d2, 2 * S * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
          double avg = 0, bx = 0;
          for (int i = 0; i < S; ++i) avg += (double)h2[i] / S, bx += (double)h2[S + i] / S;
          printf("MMA 128x%dx16 halo pattern, %s: %.1f ns/mma; TMA %.0f boxes of 16 KB meanwhile = %.1f GB/s/SM\n", bn,
                 tma ? (ST == 2 ? "2 x 16 KB TMA boxes in flight" : "4 x 16 KB TMA boxes in flight")
                     : "no TMA                       ",
                 avg / n, bx, bx * 16384 / avg);
        }
  }
  for (auto& c : cases) {
    Maps mp;
    const CUtensorMapSwizzle sw = c.box[0] * 2 >= 128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_32B;
    cuuint32_t es[4] = {1, 1, 1, 1};
    CUresult r = enc(&mp.m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, c.rank, X, c.dims, c.strides, c.box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
      printf("%s: encode failed %d\n", c.name, (int)r);
      continue;
    }
    int bytes = 2;
    for (int i = 0; i < c.rank; ++i) bytes *= c.box[i];
    for (int ST : {1, 2, 4, 8}) {
      const size_t smem = (size_t)ST * bytes + 1024;
      if (smem > 220 * 1024) continue;
      const void* kf = c.rank == 2 ? (const void*)k_tma<2> : (c.rank == 3 ? (const void*)k_tma<3> : (const void*)k_tma<4>);
      cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
      const int nbox = 400;
      for (int rep = 0; rep < 2; ++rep) {
        const int m1 = c.rank == 4 ? 0 : c.box[1], m2 = c.rank == 4 ? c.box[2] : (c.rank == 3 ? c.box[2] : 0),
                  m3 = c.rank == 4 ? c.box[3] : 0;
        if (c.rank == 2) k_tma<2><<<S, 32, smem>>>(mp, ST, nbox, bytes, c.d1, c.d2, c.d3, m1, m2, m3, d_out);
        else if (c.rank == 3) k_tma<3><<<S, 32, smem>>>(mp, ST, nbox, bytes, c.d1, c.d2, c.d3, m1, m2, m3, d_out);
        else k_tma<4><<<S, 32, smem>>>(mp, ST, nbox, bytes, c.d1, c.d2, c.d3, m1, m2, m3, d_out);
      }
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) {
        printf("%s ST=%d: %s\n", c.name, ST, cudaGetErrorString(e));
        return 1;
      }
      cudaMemcpy(h.data(), d_out, S * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
      double avg = 0;
      for (int i = 0; i < S; ++i) avg += (double)h[i] / S;
      const double ns_box = avg / nbox;
      printf("%-40s ST=%d  %7.1f ns/box  %6.1f B/clk/SM  %7.1f GB/s/SM  chip %6.2f TB/s\n", c.name, ST, ns_box,
             bytes / (ns_box * clk_khz / 1e6), bytes / ns_box, bytes / ns_box * S / 1e3);
      if (c.rank == 3) continue;
      {   // producer/consumer handoff variant
        const int m1 = c.rank == 4 ? 0 : c.box[1], m2 = c.rank == 4 ? c.box[2] : 0, m3 = c.rank == 4 ? c.box[3] : 0;
        const void* kp = c.rank == 2 ? (const void*)k_tma_pc<2> : (const void*)k_tma_pc<4>;
        cudaFuncSetAttribute(kp, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
        for (int rep = 0; rep < 2; ++rep) {
          if (c.rank == 2) k_tma_pc<2><<<S, 64, smem>>>(mp, ST, nbox, bytes, c.d1, c.d2, c.d3, m1, m2, m3, d_out);
          else k_tma_pc<4><<<S, 64, smem>>>(mp, ST, nbox, bytes, c.d1, c.d2, c.d3, m1, m2, m3, d_out);
        }
        cudaDeviceSynchronize();
        cudaMemcpy(h.data(), d_out, S * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double a2 = 0;
        for (int i = 0; i < S; ++i) a2 += (double)h[i] / S;
        printf("%-40s ST=%d  %7.1f ns/box  (producer/consumer mbarrier handoff)\n", c.name, ST, a2 / nbox);
      }
    }
  }
  return 0;
}
