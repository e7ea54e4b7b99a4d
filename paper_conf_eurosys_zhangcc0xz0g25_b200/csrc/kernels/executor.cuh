// executor.cuh -- the SM-gated persistent-CTA executor.
//
// Replaces the paper's MPS-context SM restriction:
// every tenant kernel is launched with ~S*occ CTAs; each CTA reads %smid,
// maps it to a logical SM index (probe kernel, A1) and exits at once if that
// index lies outside the kernel's range [lo, hi).  In-range CTAs pull work
// tiles from a per-launch atomic queue until it is exhausted, so a kernel runs
// on exactly the SMs it was given and partitions can change at every kernel
// boundary without MPS, MIG or any context switch (L253: BLESS needs a 50 us
// context switch here; the gate costs one %smid read).
//
// Completion protocol (per launch "slot" of a ring in device memory):
//   slot.next   tile counter (atomicAdd)
//   slot.done   CTAs that have left (atomicAdd)
//   slot.mask   logical SMs that processed >= 1 tile (R19, profiler's d)
//   slot.start  %globaltimer when tile 0 was claimed
// The CTA that brings 'done' to gridDim is the last one: it publishes
// {start, end, nsm, flags, seq} to a host-mapped stats record (poll-able
// by the host without any CUDA call) and zeroes the slot for reuse.
// Safety net: if the last CTA finds unclaimed tiles, no in-range CTA ran (the
// hardware placed every CTA elsewhere); it then processes the tiles itself and
// flags the launch (BL "fallback"), so correctness never depends on placement.
#pragma once
#include <cstdint>

namespace bless {

struct __align__(64) SlotStats {  // host-mapped, written by the last CTA
  int64_t start_gt;
  int64_t end_gt;
  uint32_t nsm;
  uint32_t flags;                  // bit0: fallback executed
  uint64_t seq;                    // written last (release)
  uint32_t mask[8];                // logical SMs that processed >= 1 tile
};

struct __align__(64) DevSlot {     // device memory, zero between launches
  uint32_t next;
  uint32_t done;
  uint32_t flags;
  uint32_t pad;
  uint32_t mask[8];
  unsigned long long start_gt;
  uint32_t pad2[2];
};

struct GateArgs {
  DevSlot* slot;
  SlotStats* stats;
  const uint8_t* lid_map;  // logical SM index per %smid (255 = unusable); null = identity
  uint64_t seq;
  uint32_t tiles;
  int32_t lo, hi;
};

#ifdef __CUDACC__
__device__ __forceinline__ uint32_t ptx_smid() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint64_t ptx_globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ int gate_lid(const GateArgs& g) {
  const uint32_t sm = ptx_smid() & 255u;
  return g.lid_map ? (int)__ldg(g.lid_map + sm) : (int)sm;
}
__device__ __forceinline__ bool gate_in_range(const GateArgs& g) {
  const int lid = gate_lid(g);
  return lid >= g.lo && lid < g.hi;
}

// Claim the next tile (call from ONE thread).  Returns -1 when exhausted.
// 'first' tracks whether this CTA already marked its SM in the mask.
__device__ __forceinline__ int gate_claim(const GateArgs& g, bool& marked) {
  const uint32_t t = atomicAdd(&g.slot->next, 1u);
  if (t >= g.tiles) return -1;
  if (t == 0) atomicExch(&g.slot->start_gt, (unsigned long long)ptx_globaltimer());
  if (!marked) {
    marked = true;
    const int lid = gate_lid(g);
    atomicOr(&g.slot->mask[(lid >> 5) & 7], 1u << (lid & 31));
  }
  return (int)t;
}

// Block-wide tile loop for simple (non warp-specialised) kernels.
// body(tile) is executed by all threads of the CTA.
template <class Body>
__device__ __forceinline__ void gate_tile_loop(const GateArgs& g, Body&& body) {
  __shared__ int s_tile;
  bool marked = false;
  for (;;) {
    if (threadIdx.x == 0) s_tile = gate_claim(g, marked);
    __syncthreads();
    const int t = s_tile;
    __syncthreads();
    if (t < 0) break;
    body(t);
  }
}

// Exit protocol.  Returns true if THIS CTA must run the work loop as the
// fallback (see header).  All threads of the CTA must call it.
__device__ __forceinline__ bool gate_leave(const GateArgs& g, int& is_last) {
  __shared__ int s_flag;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const uint32_t nblk = gridDim.x * gridDim.y * gridDim.z;
    const uint32_t prev = atomicAdd(&g.slot->done, 1u);
    int flag = 0;
    if (prev == nblk - 1) {
      const uint32_t nxt = atomicAdd(&g.slot->next, 0u);
      flag = (nxt < g.tiles) ? 2 : 1;
    }
    s_flag = flag;
  }
  __syncthreads();
  is_last = s_flag != 0;
  return s_flag == 2;
}

// Called by the last CTA (after any fallback work): publish and reset.
__device__ __forceinline__ void gate_finalize(const GateArgs& g, bool fallback) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    DevSlot* s = g.slot;
    uint32_t nsm = 0;
    volatile SlotStats* out = g.stats;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const uint32_t w = ((volatile uint32_t*)s->mask)[i];
      out->mask[i] = w;
      nsm += __popc(w);
    }
    const uint64_t end = ptx_globaltimer();
    uint64_t st = *(volatile unsigned long long*)&s->start_gt;
    if (st == 0) st = end;
    out->start_gt = (int64_t)st;
    out->end_gt = (int64_t)end;
    out->nsm = nsm;
    out->flags = fallback ? 1u : 0u;
    __threadfence_system();
    out->seq = g.seq;
    // reset the slot for its next use (ring reuse is >= 64K launches later)
    s->next = 0;
    s->done = 0;
    s->flags = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) s->mask[i] = 0;
    s->start_gt = 0;
    __threadfence();
  }
}

// The canonical gated kernel body for tile-loop ops: Op::tile(params, t, smem).
template <class Op>
__device__ __forceinline__ void gated_run(const typename Op::Params& p, const GateArgs& g, unsigned char* smem) {
  if (gate_in_range(g)) gate_tile_loop(g, [&](int t) { Op::tile(p, t, smem); });
  int last = 0;
  const bool fb = gate_leave(g, last);
  if (fb) gate_tile_loop(g, [&](int t) { Op::tile(p, t, smem); });
  if (last) gate_finalize(g, fb);
}
#endif

}  // namespace bless
