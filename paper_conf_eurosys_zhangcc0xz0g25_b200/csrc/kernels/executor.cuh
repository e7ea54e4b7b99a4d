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
// Per-launch state lives in a ring of "slots" (device memory):
//   slot.ctr   64-bit word: low 32 bits = tile counter (claims), high 32 bits
//              = CTAs that have left.  One atomic per CTA on exit returns both,
//              so the last CTA learns "am I last" and "were all tiles claimed"
//              in a single round trip.
// and a ring of stats records (device memory, mirrored to the host by
// copy-engine reads -- no SM ever waits on PCIe):
//   stats.start  %globaltimer when tile 0 was claimed (written by that CTA)
//   stats.mask   logical SMs that processed >= 1 tile (atomicOr per CTA; R19)
//   stats.end / flags / seq   written by the last CTA (seq last, after a fence)
// The last CTA also zeroes the mask of the stats record it will reuse
// DeviceRT::ahead() launches later and resets its slot word.
// Safety net: if the last CTA finds unclaimed tiles, no in-range CTA ran (the
// hardware placed every CTA elsewhere); it then processes the tiles itself and
// flags the launch ("fallback"), so correctness never depends on placement.
//
// Light exit: most launches (a request's middle kernels) skip the exit
// protocol (stamp = 0): no per-CTA atomic, no last-CTA publish, so the grid
// completes as soon as its last tile's stores are issued (the exit protocol
// was 1.5-2.4 us of a batch-1 kernel's critical path, profiles/round1/
// tctrace_*).  Their end time is stamped by the successor on the same stream
// when its griddepcontrol.wait returns (prev_stats); the slot and stats record
// reuse is handled ahead of time by the tile-0 claimer.  Launches whose
// completion the host must observe (a request's first/last kernel, the last
// kernel of a tenant's chain in a squad, profiling) use the full protocol.
// No tile is ever lost without the fallback: out-of-range CTAs linger and
// help after a timeout, so every queue drains.
//
// Programmatic dependent launch: kernels are launched with programmatic stream
// serialization; a CTA waits (griddepcontrol.wait) only right before touching
// data produced by the previous kernel, and signals its dependents as soon as
// the tile queue is exhausted, so a kernel's launch and prologue overlap the
// tail of its predecessor on the tenant's stream.
#pragma once
#include <cstdint>
#include <cstdlib>

namespace bless {

struct __align__(64) SlotStats {
  int64_t start_gt;
  int64_t end_gt;
  uint32_t nsm;        // unused on device (host computes popcount of mask)
  uint32_t flags;      // bit0: fallback executed
  uint64_t seq;        // written last, after a device-scope fence
  uint32_t mask[8];    // logical SMs that processed >= 1 tile
};

struct __align__(16) DevSlot {  // device memory, zero between launches
  unsigned long long ctr;       // [31:0] claims, [63:32] CTAs done
  unsigned long long done;      // units finished (software dependency, count_done launches)
};


struct GateArgs {
  DevSlot* slot;
  SlotStats* stats;        // this launch's record
  SlotStats* stats_ahead;  // record of launch seq + ahead (flags/mask zeroed here; ahead = ring / 2)
  DevSlot* slot_ahead;     // slot of launch seq + ahead (zeroed here)
  SlotStats* prev_stats;   // light predecessor on the stream (its end stamp is written here) or null
  const uint8_t* lid_map;  // logical SM index per %smid (255 = unusable); null = identity
  uint64_t seq;
  uint32_t tiles;
  int32_t lo, hi;
  uint32_t stamp;          // 1: full exit protocol (last CTA publishes end + seq); 0: light exit
  uint32_t linger_ns;      // bounded wait of out-of-range CTAs (default 30 us; BLESS_LINGER_NS, tests)
  // Software dependency (tcgen05 GEMM/conv chains): a
  // count_done launch adds 1 to slot->done after each finished unit (its
  // stores fenced first); a launch with dep_ctr set waits for its stream
  // predecessor's counter to reach dep_total instead of griddepcontrol.wait
  // (the predecessor's last CTA exit, grid completion and memory flush are
  // off the critical path).
  const unsigned long long* dep_ctr;
  uint32_t dep_total;
  uint32_t count_done;
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
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ int gate_lid(const GateArgs& g) {
  const uint32_t sm = ptx_smid() & 255u;
  return g.lid_map ? (int)__ldg(g.lid_map + sm) : (int)sm;
}
__device__ __forceinline__ bool gate_in_range(const GateArgs& g) {
  const int lid = gate_lid(g);
  return lid >= g.lo && lid < g.hi;
}

// Wait for the data of the previous kernel on the stream: the software
// dependency when the predecessor counts its finished units (every lane
// acquires the counter; the proxy fence orders the TMA loads that follow),
// else griddepcontrol.wait.  Called by whole warps.
__device__ __forceinline__ void dep_wait(const GateArgs& g) {
  if (g.dep_ctr == nullptr) {
    pdl_wait();
    return;
  }
  // every lane polls (one broadcast load): the loop stays warp-uniform, which
  // keeps ptxas on the uniform datapath for the TMA/MMA issue around it
  uint64_t t0 = 0;
  bool timed_out = false;
  for (int i = 0;; ++i) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(g.dep_ctr) : "memory");
    if (__all_sync(0xffffffffu, v >= g.dep_total)) break;
    // safety net: a counter that does not reach its total within 5 ms (a
    // host bookkeeping error) falls back to the hardware dependency, flagged
    if ((i & 63) == 63) {
      const uint64_t now = __shfl_sync(0xffffffffu, ptx_globaltimer(), 0);
      if (!t0) {
        t0 = now;
      } else if (now - t0 > 5000000ull) {
        timed_out = true;
        break;
      }
    }
    __nanosleep(32);
  }
  if (timed_out) {
    if ((threadIdx.x & 31) == 0) atomicOr(&g.stats->flags, 4u);
    pdl_wait();
  }
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

// Claim the next tile (call from ONE thread).  Returns -1 when exhausted.
// 'marked' tracks whether this CTA already set its SM bit in the mask.
// The claimer of tile 0 stamps the start, zeroes the slot and the stats
// flags/mask of the launch `ahead` seqs later (no CTA of that ring position's
// previous launch can still run), and -- if it claims after
// griddepcontrol.wait (after_wait) -- writes the end stamp of a light
// predecessor on the stream, which completed exactly when that wait returned.
__device__ __forceinline__ void gate_prev_end(const GateArgs& g, int64_t now) {
  if (g.prev_stats) g.prev_stats->end_gt = now;
}
__device__ __forceinline__ int gate_claim(const GateArgs& g, bool& marked, bool after_wait = true) {
  const uint32_t t = (uint32_t)atomicAdd(&g.slot->ctr, 1ull);
  if (t >= g.tiles) return -1;
  if (t == 0) {
    const int64_t now = (int64_t)ptx_globaltimer();
    g.stats->start_gt = now;
    g.slot_ahead->ctr = 0ull;
    g.slot_ahead->done = 0ull;
    g.stats_ahead->flags = 0u;
    uint4* fm = reinterpret_cast<uint4*>(g.stats_ahead->mask);
    fm[0] = make_uint4(0, 0, 0, 0);
    fm[1] = make_uint4(0, 0, 0, 0);
    if (after_wait) gate_prev_end(g, now);
  }
  if (!marked) {
    marked = true;
    const int lid = gate_lid(g);
    atomicOr(&g.stats->mask[(lid >> 5) & 7], 1u << (lid & 31));
  }
  return (int)t;
}

// Block-wide tile loop for simple (non warp-specialised) kernels.
// body(tile) is executed by all threads of the CTA.  (Measured on B200: a
// variant that claimed the first tile before griddepcontrol.wait, or issued
// the next claim inside the previous body, made LayerNorm 384x1024 slower,
// 8.8 -> 11.0 us, with its 48 tiles landing on 17 SMs instead of 24 --
// profiles/round1/ln_executor_ab.txt.)
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

// Out-of-range CTAs linger until some in-range CTA has claimed a tile (or a
// bounded timeout): otherwise, when the kernel's own SMs are still busy (e.g.
// its predecessor under programmatic dependent launch, or another tenant's
// CTAs), every CTA of the grid could be placed out of range and leave, and
// the work would fall back to a single CTA.  The timeout breaks mutual waits
// between tenants.
// Under programmatic dependent launch the busy in-range SMs are most often
// held by this kernel's own predecessor on the stream, so a lingering CTA
// first waits for that grid to complete (it cannot deadlock: all of the
// predecessor's CTAs are resident when dependents launch) and only then starts
// the bounded wait for an in-range CTA.
// Grids are sized to the kernel's full occupancy (S x blocks/SM), so lingering
// CTAs on out-of-range SMs can never absorb the whole grid: some CTAs stay
// queued until the window frees up.  If no in-range CTA has claimed a tile
// when the bounded wait expires (e.g. two tenants' lingering CTAs blocking
// each other's windows), the CTA returns true and helps drain the queue (a
// bounded, flagged confinement violation instead of a stalled kernel).
constexpr uint64_t kLingerNs = 30000;   // default GateArgs::linger_ns
__device__ __forceinline__ bool gate_linger(const GateArgs& g) {
  __shared__ int s_steal;
  if (threadIdx.x == 0) {
    int steal = 0;
    if (g.tiles > 0 && g.lo < g.hi) {
      pdl_wait();
      const uint64_t t0 = ptx_globaltimer();
      for (;;) {
        const unsigned long long c = *reinterpret_cast<volatile unsigned long long*>(&g.slot->ctr);
        if ((uint32_t)c != 0u) break;
        if (ptx_globaltimer() - t0 > g.linger_ns) {
          steal = 1;
          break;
        }
        __nanosleep(256);
      }
      if (steal) atomicOr(&g.stats->flags, 2u);
    }
    s_steal = steal;
  }
  __syncthreads();
  return s_steal != 0;
}

// Exit protocol.  Returns true if THIS CTA must run the work loop as the
// fallback (see header).  All threads of the CTA must call it.
__device__ __forceinline__ bool gate_leave(const GateArgs& g, int& is_last) {
  __shared__ int s_flag;
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t nblk = gridDim.x * gridDim.y * gridDim.z;
    const unsigned long long prev = atomicAdd(&g.slot->ctr, 1ull << 32);
    int flag = 0;
    if ((uint32_t)(prev >> 32) == nblk - 1) flag = ((uint32_t)prev < g.tiles) ? 2 : 1;
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
    const uint64_t end = ptx_globaltimer();
    SlotStats* out = g.stats;
    out->end_gt = (int64_t)end;
    if (g.tiles == 0) out->start_gt = (int64_t)end;
    if (fallback) atomicOr(&out->flags, 1u);
    if (g.tiles == 0) {   // nothing was claimed: zero ahead here (marker launches)
      g.slot_ahead->ctr = 0ull;
      g.slot_ahead->done = 0ull;
      g.stats_ahead->flags = 0u;
      uint4* fm = reinterpret_cast<uint4*>(g.stats_ahead->mask);
      fm[0] = make_uint4(0, 0, 0, 0);
      fm[1] = make_uint4(0, 0, 0, 0);
    }
    g.slot->ctr = 0ull;
    __threadfence();
    *reinterpret_cast<volatile uint64_t*>(&out->seq) = g.seq;
  }
}

// The canonical gated kernel body for tile-loop ops: Op::tile(params, t, smem).
template <class Op>
__device__ __forceinline__ void gated_run(const typename Op::Params& p, const GateArgs& g, unsigned char* smem) {
  if (gate_in_range(g) || gate_linger(g)) {
    pdl_wait();
    gate_tile_loop(g, [&](int t) { Op::tile(p, t, smem); });
  }
  pdl_trigger();
  if (!g.stamp) return;   // light exit (see header)
  int last = 0;
  const bool fb = gate_leave(g, last);
  if (fb) {
    pdl_wait();
    gate_tile_loop(g, [&](int t) { Op::tile(p, t, smem); });
  }
  if (last) gate_finalize(g, fb);
}
#endif

// Host: launch with programmatic stream serialization (PDL) unless disabled.
extern int g_use_pdl;
#ifdef __CUDACC__
// Grid = S x (resident blocks per SM for this kernel), capped at 8 per SM and
// at the kernel's own cap (small-work SIMT kernels run faster with fewer CTAs:
// fewer claims on the tile queue and fewer idle CTAs to launch and retire).
inline int full_occupancy_grid(const void* fn, int block, size_t smem, int S, int max_occ = 8) {
  int occ = 1;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, block, smem) != cudaSuccess || occ < 1) occ = 1;
  static const int cap = [] {   // BLESS_MAX_OCC: blocks-per-SM cap (sweeps; default 8)
    const char* e = std::getenv("BLESS_MAX_OCC");
    const int v = e ? std::atoi(e) : 8;
    return v < 1 ? 1 : (v > 8 ? 8 : v);
  }();
  const int c = cap < max_occ ? cap : max_occ;
  return S * (occ > c ? c : occ);
}
inline cudaError_t launch_kernel(const void* fn, dim3 grid, dim3 block, size_t smem, cudaStream_t st, void** args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = g_use_pdl ? 1 : 0;
  return cudaLaunchKernelExC(&cfg, fn, args);
}
#endif

}  // namespace bless
