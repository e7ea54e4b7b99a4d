// cuda_rt.cu -- see cuda_rt.hpp.
#include "cuda_rt.hpp"

#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <vector>
#include <atomic>
#include <chrono>
#include <cstring>
#include <cstdlib>
#include <thread>

#include "../kernels/executor.cuh"

namespace bless {

int g_use_pdl = 1;

static int64_t host_now_ns() {
  return std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

#define RT_CHECK(call)                                                          \
  do {                                                                          \
    cudaError_t e_ = (call);                                                    \
    if (e_ != cudaSuccess) {                                                    \
      err = std::string(#call) + ": " + cudaGetErrorString(e_);                 \
      return false;                                                             \
    }                                                                           \
  } while (0)

// ---------------------------------------------------------------- probe kernels (A1)
__global__ void k_probe_smid(unsigned* seen, unsigned* nsmid_out) {
  const uint32_t sm = ptx_smid();
  if (threadIdx.x == 0) {
    atomicOr(&seen[(sm >> 5) & 7], 1u << (sm & 31));
    uint32_t n;
    asm volatile("mov.u32 %0, %%nsmid;" : "=r"(n));
    atomicMax(nsmid_out, n);
  }
}

__global__ void __cluster_dims__(2, 1, 1) k_probe_pairs(int* out) {
  if (threadIdx.x == 0) out[blockIdx.x] = (int)ptx_smid();
}

__global__ void k_clock(unsigned long long* out) {
  if (threadIdx.x == 0) {
    const unsigned long long t = ptx_globaltimer();
    *(volatile unsigned long long*)out = t;
    __threadfence_system();
  }
}

__global__ void k_gt_res(long long* out) {
  uint64_t prev = ptx_globaltimer();
  long long best = 1LL << 40;
  for (int i = 0; i < 20000; ++i) {
    const uint64_t t = ptx_globaltimer();
    if (t != prev) {
      best = min(best, (long long)(t - prev));
      prev = t;
    }
  }
  *out = best;
}

// ---------------------------------------------------------------- kernel dispatch
bool build_kernel(const bl_op& op, const DeviceCaps& caps, KernelDesc& out, std::string& err) {
  if (op.kind == BL_OP_VIRTUAL) { err = "virtual op on a device ctx"; return false; }
  std::string e2;
  if (build_attn_tc(op, caps, out, e2)) return true;
  if (!e2.empty()) { err = e2; return false; }
  if (build_nn(op, caps, out, e2)) return true;
  if (!e2.empty()) { err = e2; return false; }
  if (op.dtype == BL_BF16 && op.kind == BL_OP_GEMM && op.dims[0] <= 8) {
    if (build_gemv_tma(op, caps, out, e2)) return true;
    if (!e2.empty()) { err = e2; return false; }
  }
  if (op.dtype == BL_BF16 && (op.kind == BL_OP_GEMM || op.kind == BL_OP_CONV)) {
    if (build_tc_gemm(op, caps, out, e2)) return true;
    if (!e2.empty()) { err = e2; return false; }
  }
  return build_simt(op, caps, out, err);
}

// ---------------------------------------------------------------- DeviceRT
std::unique_ptr<DeviceRT> DeviceRT::create(int device, void* ws, size_t ws_bytes, std::string& err) {
  std::unique_ptr<DeviceRT> rt(new DeviceRT());
  rt->device_ = device;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || device < 0 || device >= ndev) {
    err = std::string("no CUDA device ") + std::to_string(device) + " (" + cudaGetErrorString(e) + ")";
    return nullptr;
  }
  if (cudaSetDevice(device) != cudaSuccess) { err = "cudaSetDevice"; return nullptr; }
  cudaDeviceProp prop{};
  cudaGetDeviceProperties(&prop, device);
  rt->info_.device = device;
  rt->info_.sm_count = prop.multiProcessorCount;
  rt->info_.cc_major = prop.major;
  rt->info_.cc_minor = prop.minor;
  rt->info_.l2_bytes = prop.l2CacheSize;
  rt->info_.smem_per_block_optin = (int64_t)prop.sharedMemPerBlockOptin;
  rt->caps_.S = prop.multiProcessorCount;
  rt->caps_.cc_major = prop.major;
  rt->caps_.cc_minor = prop.minor;
  rt->caps_.smem_optin = (int)prop.sharedMemPerBlockOptin;
  if (const char* e = std::getenv("BLESS_STATS_RING_LOG2")) {
    const int l2 = std::atoi(e);
    if (l2 >= 10 && l2 <= 22) rt->ring_ = 1ull << l2;
  }
  rt->ahead_ = rt->ring_ / 2;
  const uint64_t kSlotRing = rt->ring_;
  const size_t slot_bytes = kSlotRing * sizeof(DevSlot);
  if (ws && ws_bytes >= slot_bytes) {
    rt->slots_ = ws;
    rt->own_slots_ = false;
  } else {
    if (cudaMalloc(&rt->slots_, slot_bytes) != cudaSuccess) { err = "cudaMalloc slots"; return nullptr; }
    rt->own_slots_ = true;
  }
  if (cudaMemset(rt->slots_, 0, slot_bytes) != cudaSuccess) { err = "memset slots"; return nullptr; }
  // stats ring in device memory + pinned host mirror refreshed by async copies
  if (cudaMalloc(&rt->stats_dev_, kSlotRing * sizeof(SlotStats)) != cudaSuccess ||
      cudaMemset(rt->stats_dev_, 0, kSlotRing * sizeof(SlotStats)) != cudaSuccess) {
    err = "cudaMalloc stats";
    return nullptr;
  }
  if (cudaHostAlloc(&rt->stats_host_, kSlotRing * sizeof(SlotStats), cudaHostAllocDefault) != cudaSuccess) {
    err = "cudaHostAlloc stats mirror";
    return nullptr;
  }
  std::memset(rt->stats_host_, 0, kSlotRing * sizeof(SlotStats));
  if (cudaStreamCreateWithPriority((cudaStream_t*)&rt->reader_, cudaStreamNonBlocking, 0) != cudaSuccess ||
      cudaEventCreateWithFlags((cudaEvent_t*)&rt->reader_ev_, cudaEventDisableTiming) != cudaSuccess) {
    err = "reader stream";
    return nullptr;
  }
  if (const char* e = std::getenv("BLESS_PDL")) g_use_pdl = std::atoi(e) != 0;
  rt->linger_ns_ = (uint32_t)kLingerNs;
  if (const char* e = std::getenv("BLESS_LINGER_NS")) rt->linger_ns_ = (uint32_t)std::max(0, std::atoi(e));
  if (const char* e = std::getenv("BLESS_SWDEP")) rt->swdep_ = std::atoi(e) != 0;
  if (const char* e = std::getenv("BLESS_TC_AUTOTUNE")) rt->autotune_ = std::atoi(e) != 0;
  if (const char* e = std::getenv("BLESS_TC_TUNE_FILE")) {   // "sig bn splits" lines, appended as tuned
    rt->tune_file_ = e;
    if (FILE* f = std::fopen(e, "r")) {
      char sig[512];
      int bn = 0, sp = 0, bk = 0, halo = 0, mt = 0;
      while (std::fscanf(f, "%511s %d %d %d %d %d", sig, &bn, &sp, &bk, &halo, &mt) == 6)
        rt->tune_cache_[sig] = TcChoice{bn, sp, bk, halo, mt};
      std::fclose(f);
    }
  }
  if (!rt->probe(err)) return nullptr;
  if (!rt->calibrate_clock(err)) return nullptr;
  return rt;
}

DeviceRT::~DeviceRT() {
  cudaSetDevice(device_);
  cudaDeviceSynchronize();
  if (own_slots_ && slots_) cudaFree(slots_);
  if (stats_dev_) cudaFree(stats_dev_);
  if (stats_host_) cudaFreeHost(stats_host_);
  if (reader_ev_) cudaEventDestroy((cudaEvent_t)reader_ev_);
  if (reader_) cudaStreamDestroy((cudaStream_t)reader_);
  if (lid_map_dev_) cudaFree(lid_map_dev_);
  for (auto& k : kernels_)
    if (k && k->owned) cudaFree(k->owned);
  if (tune_stream_) cudaStreamDestroy((cudaStream_t)tune_stream_);
}

bool DeviceRT::set_device() { return cudaSetDevice(device_) == cudaSuccess; }

bool DeviceRT::probe(std::string& err) {
  unsigned* d = nullptr;
  RT_CHECK(cudaMalloc(&d, 64));
  RT_CHECK(cudaMemset(d, 0, 64));
  const int S = info_.sm_count;
  k_probe_smid<<<S * 16, 64>>>(d, d + 8);
  RT_CHECK(cudaGetLastError());
  unsigned h[9];
  RT_CHECK(cudaMemcpy(h, d, 36, cudaMemcpyDeviceToHost));
  std::vector<int> smids;
  for (int i = 0; i < 256; ++i)
    if (h[i >> 5] & (1u << (i & 31))) smids.push_back(i);
  info_.max_smid = (int)h[8] - 1;
  std::memset(info_.smid_to_lid, 255, 256);
  // Logical order = ascending %smid (TPC siblings are adjacent ids).
  for (size_t i = 0; i < smids.size(); ++i) info_.smid_to_lid[smids[i]] = (uint8_t)i;
  identity_map_ = true;
  for (size_t i = 0; i < smids.size(); ++i)
    if (smids[i] != (int)i) identity_map_ = false;
  if ((int)smids.size() != S) {
    err = "probe saw " + std::to_string(smids.size()) + " SMs, expected " + std::to_string(S);
    cudaFree(d);
    return false;
  }
  RT_CHECK(cudaMalloc(&lid_map_dev_, 256));
  RT_CHECK(cudaMemcpy(lid_map_dev_, info_.smid_to_lid, 256, cudaMemcpyHostToDevice));
  // TPC pairs via 2-CTA clusters (informational: siblings whose ids differ by one).
  int* pr = nullptr;
  const int npairs = (S / 2) * 2;
  RT_CHECK(cudaMalloc(&pr, sizeof(int) * npairs));
  k_probe_pairs<<<npairs, 32>>>(pr);
  if (cudaGetLastError() == cudaSuccess) {
    std::vector<int> hp(npairs);
    cudaMemcpy(hp.data(), pr, sizeof(int) * npairs, cudaMemcpyDeviceToHost);
    int ok = 0;
    for (int i = 0; i + 1 < npairs; i += 2)
      if ((hp[i] ^ hp[i + 1]) == 1) ok++;
    info_.tpc_pairs_found = ok;
  }
  cudaFree(pr);
  long long* r = nullptr;
  RT_CHECK(cudaMalloc(&r, 8));
  k_gt_res<<<1, 1>>>(r);
  long long res = 0;
  RT_CHECK(cudaMemcpy(&res, r, 8, cudaMemcpyDeviceToHost));
  info_.globaltimer_res_ns = res;
  cudaFree(r);
  cudaFree(d);
  return true;
}

bool DeviceRT::calibrate_clock(std::string& err) {
  unsigned long long* hp = nullptr;
  RT_CHECK(cudaHostAlloc((void**)&hp, 64, cudaHostAllocMapped));
  unsigned long long* dp = nullptr;
  RT_CHECK(cudaHostGetDevicePointer((void**)&dp, hp, 0));
  cudaStream_t s;
  RT_CHECK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  int64_t best_span = INT64_MAX, best_off = 0;
  for (int it = 0; it < 9; ++it) {
    *(volatile unsigned long long*)hp = 0;
    const int64_t t0 = host_now_ns();
    k_clock<<<1, 32, 0, s>>>(dp);
    while (*(volatile unsigned long long*)hp == 0) {
    }
    const int64_t t1 = host_now_ns();
    const int64_t gt = (int64_t) * (volatile unsigned long long*)hp;
    // the kernel ran between t0 + launch latency and t1 - visibility latency;
    // attribute the stamp to 3/4 of the span (launch latency dominates).
    const int64_t est = t0 + (t1 - t0) * 3 / 4;
    if (t1 - t0 < best_span) {
      best_span = t1 - t0;
      best_off = gt - est;
    }
  }
  cudaStreamSynchronize(s);
  cudaStreamDestroy(s);
  cudaFreeHost(hp);
  info_.clock_offset_ns = best_off;
  return true;
}

// Shared-memory carveout of every tenant kernel (BLESS_CARVEOUT = percent of
// the unified L1/shared array given to shared memory; unset = driver default).
// One carveout for all kernels means an SM never has to drain and
// reconfigure L1/shared between a tcgen05 kernel (~100 KB of shared memory)
// and a SIMT kernel (a few KB) of the same or another tenant.
static void apply_carveout(const void* fn) {
  static const int pct = [] {
    const char* e = std::getenv("BLESS_CARVEOUT");
    return e ? std::atoi(e) : -1;
  }();
  if (fn && pct >= 0 && pct <= 100) cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
}

int DeviceRT::add_kernel(const bl_op& op, std::string& err) {
  std::unique_ptr<KernelDesc> kd(new KernelDesc());
  if (!build_kernel(op, caps_, *kd, err)) return -1;
  apply_carveout(kd->kernel_fn);
  // grid = S x (resident blocks per SM): see gate_linger in executor.cuh
  if (kd->kernel_fn) {
    kd->grid = full_occupancy_grid(kd->kernel_fn, kd->block, (size_t)kd->smem, caps_.S, kd->max_occ);
    kd->grid_full = full_occupancy_grid(kd->kernel_fn, kd->block, (size_t)kd->smem, caps_.S);
    kd->S = caps_.S;
  }
  if (kd->choice_bn && autotune_ && !std::getenv("BLESS_TC_CFG")) {
    const std::string sig = tc_signature(op);
    auto it = tune_cache_.find(sig);
    if (it != tune_cache_.end()) {
      if (it->second.bn != kd->choice_bn || it->second.splits != kd->choice_splits ||
          it->second.bk != kd->choice_bk || it->second.halo != kd->choice_halo ||
          it->second.mt != kd->choice_mt) {
        std::unique_ptr<KernelDesc> k2(new KernelDesc());
        std::string e2;
        if (build_tc_gemm(op, caps_, *k2, e2, &it->second)) {
          k2->grid = full_occupancy_grid(k2->kernel_fn, k2->block, (size_t)k2->smem, caps_.S, k2->max_occ);
          k2->grid_full = full_occupancy_grid(k2->kernel_fn, k2->block, (size_t)k2->smem, caps_.S);
          k2->S = caps_.S;
          if (kd->owned) cudaFree(kd->owned);
          kd = std::move(k2);
        }
      }
    } else {
      if (!autotune_tc(op, kd, err)) return -1;
      tune_cache_[sig] = TcChoice{kd->choice_bn, kd->choice_splits, kd->choice_bk, kd->choice_halo, kd->choice_mt};
      if (!tune_file_.empty()) {
        if (FILE* f = std::fopen(tune_file_.c_str(), "a")) {
          std::fprintf(f, "%s %d %d %d %d %d\n", sig.c_str(), kd->choice_bn, kd->choice_splits, kd->choice_bk,
                       kd->choice_halo, kd->choice_mt);
          std::fclose(f);
        }
      }
    }
  }
  apply_carveout(kd->kernel_fn);
  kernels_.push_back(std::move(kd));
  return (int)kernels_.size() - 1;
}

// Shape signature of a tc op for the tuning cache (pointers excluded).
std::string DeviceRT::tc_signature(const bl_op& op) const {
  // "v2": tune files since the autotuner also picks BK (older lines never match)
  std::string s = "v5k" + std::to_string(op.kind) + "_t" + std::to_string(op.dtype) + "_r" + (op.ptr[4] ? "1" : "0");
  for (int i = 0; i < 12; ++i) s += "_" + std::to_string(op.dims[i]);
  return s;
}

// Registration-time choice of the tcgen05 tile configuration (part of the
// offline profiling stage): every candidate is timed like
// the profiler times a kernel (back-to-back launches on one stream, CUDA
// events, all S SMs) on the layer's own buffers; the fastest wins, and within
// 3 % of it the one with fewer tiles (smaller d leaves more SMs to co-runners).
bool DeviceRT::autotune_tc(const bl_op& op, std::unique_ptr<KernelDesc>& best, std::string& err) {
  TcChoice cand[32];
  const int nc = tc_candidates(op, caps_, cand, 32);
  if (nc <= 1) return true;
  if (!tune_stream_ && cudaStreamCreateWithFlags((cudaStream_t*)&tune_stream_, cudaStreamNonBlocking) != cudaSuccess) {
    err = "autotune stream";
    return false;
  }
  int64_t best_ns = 0;
  {
    kernels_.push_back(std::move(best));
    const int h = (int)kernels_.size() - 1;
    const bool ok = profile(h, caps_.S, 4, tune_stream_, &best_ns, nullptr, err);
    best = std::move(kernels_.back());
    kernels_.pop_back();
    if (!ok) return false;
  }
  for (int i = 0; i < nc; ++i) {
    if (cand[i].bn == best->choice_bn && cand[i].splits == best->choice_splits && cand[i].bk == best->choice_bk &&
        cand[i].halo == best->choice_halo && (cand[i].mt ? cand[i].mt : 128) == best->choice_mt)
      continue;
    std::unique_ptr<KernelDesc> kd(new KernelDesc());
    std::string e2;
    if (!build_tc_gemm(op, caps_, *kd, e2, &cand[i])) continue;
    if (kd->choice_bn == best->choice_bn && kd->choice_splits == best->choice_splits &&
        kd->choice_bk == best->choice_bk && kd->choice_halo == best->choice_halo && kd->choice_mt == best->choice_mt) {
      if (kd->owned) cudaFree(kd->owned);
      continue;
    }
    kd->grid = full_occupancy_grid(kd->kernel_fn, kd->block, (size_t)kd->smem, caps_.S, kd->max_occ);
    kd->grid_full = full_occupancy_grid(kd->kernel_fn, kd->block, (size_t)kd->smem, caps_.S);
    kd->S = caps_.S;
    kernels_.push_back(std::move(kd));
    const int h = (int)kernels_.size() - 1;
    int64_t ns = 0;
    const bool ok = profile(h, caps_.S, 4, tune_stream_, &ns, nullptr, err);
    kd = std::move(kernels_.back());
    kernels_.pop_back();
    if (!ok) {
      if (kd->owned) cudaFree(kd->owned);
      return false;
    }
    const bool better = (double)ns < 0.97 * (double)best_ns ||
                        ((double)ns <= 1.03 * (double)best_ns && kd->tiles < best->tiles);
    std::unique_ptr<KernelDesc>& loser = better ? best : kd;
    if (better) best_ns = ns;
    if (loser->owned) {
      cudaStreamSynchronize((cudaStream_t)tune_stream_);
      cudaFree(loser->owned);
      loser->owned = nullptr;
    }
    if (better) best = std::move(kd);
  }
  return true;
}

GateArgs DeviceRT::make_gate(uint64_t seq, uint32_t tiles, int lo, int hi, bool stamp, uint64_t prev_light) const {
  GateArgs g;
  const uint64_t R = ring_;
  g.slot = reinterpret_cast<DevSlot*>(slots_) + seq % R;
  g.stats = reinterpret_cast<SlotStats*>(stats_dev_) + seq % R;
  g.stats_ahead = reinterpret_cast<SlotStats*>(stats_dev_) + (seq + ahead_) % R;
  g.slot_ahead = reinterpret_cast<DevSlot*>(slots_) + (seq + ahead_) % R;
  g.prev_stats = prev_light ? reinterpret_cast<SlotStats*>(stats_dev_) + prev_light % R : nullptr;
  g.lid_map = identity_map_ ? nullptr : lid_map_dev_;
  g.seq = seq;
  g.tiles = tiles;
  g.lo = lo;
  g.hi = hi;
  g.stamp = stamp ? 1u : 0u;
  g.linger_ns = linger_ns_;
  g.dep_ctr = nullptr;
  g.dep_total = 0;
  g.count_done = 0;
  return g;
}

uint64_t DeviceRT::launch(int h, int lo, int hi, void* stream, std::string& err, bool stamp) {
  const KernelDesc& kd = *kernels_[h];
  const uint64_t seq = ++seq_;
  const GateArgs g = make_gate(seq, kd.tiles, lo, hi, stamp, 0);
  const cudaError_t e = kd.launch(kd, g, (cudaStream_t)stream);
  if (e != cudaSuccess) {
    err = std::string("launch ") + kd.family + ": " + cudaGetErrorString(e);
    return 0;
  }
  return seq;
}

bool DeviceRT::launch_seq(int h, uint64_t seq, int lo, int hi, void* stream, std::string& err, bool stamp,
                          uint64_t prev_light, uint64_t dep_seq, uint32_t dep_total) {
  const KernelDesc& kd = *kernels_[h];
  GateArgs g = make_gate(seq, kd.tiles, lo, hi, stamp, prev_light);
  if (counts(h)) {
    g.count_done = 1u;
    if (dep_seq) {
      g.dep_ctr = &(reinterpret_cast<DevSlot*>(slots_) + dep_seq % ring_)->done;
      g.dep_total = dep_total;
    }
  }
  const cudaError_t e = kd.launch(kd, g, (cudaStream_t)stream);
  if (e != cudaSuccess) {
    err = std::string("launch ") + kd.family + ": " + cudaGetErrorString(e);
    return false;
  }
  return true;
}

__global__ void k_marker(const GateArgs g);

bool DeviceRT::launch_marker_seq(uint64_t seq, void* stream, std::string& err) {
  GateArgs g = make_gate(seq, 0, 0, 0);
  g.lid_map = nullptr;
  k_marker<<<1, 32, 0, (cudaStream_t)stream>>>(g);
  const cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    err = std::string("marker: ") + cudaGetErrorString(e);
    return false;
  }
  return true;
}

__global__ void k_marker(const GateArgs g) {
  // zero tiles: the single CTA is the last one and publishes the stamps
  int last = 0;
  const bool fb = gate_leave(g, last);
  if (last) gate_finalize(g, fb);
}

uint64_t DeviceRT::launch_marker(void* stream, std::string& err) {
  const uint64_t seq = ++seq_;
  GateArgs g = make_gate(seq, 0, 0, 0);
  g.lid_map = nullptr;
  k_marker<<<1, 32, 0, (cudaStream_t)stream>>>(g);
  const cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    err = std::string("marker: ") + cudaGetErrorString(e);
    return 0;
  }
  return seq;
}

// ---------------------------------------------------------------- diagnostics
__global__ void k_empty() {}
__global__ void k_gate_only(const GateArgs g, int publish) {
  __shared__ int s_t;
  bool marked = false;
  if (gate_in_range(g)) {
    pdl_wait();
    for (;;) {
      if (threadIdx.x == 0) s_t = gate_claim(g, marked);
      __syncthreads();
      const int t = s_t;
      __syncthreads();
      if (t < 0) break;
    }
  }
  pdl_trigger();
  int last = 0;
  const bool fb = gate_leave(g, last);
  if (last) {
    if (publish) {
      gate_finalize(g, fb);
    } else if (threadIdx.x == 0) {
      g.slot->ctr = 0ull;
    }
  }
}

bool DeviceRT::overhead(int variant, int reps, int64_t* ns_out, std::string& err) {
  cudaStream_t s = nullptr;
  RT_CHECK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t e0, e1;
  RT_CHECK(cudaEventCreate(&e0));
  RT_CHECK(cudaEventCreate(&e1));
  const int S = info_.sm_count;
  const bool host_time = (variant & 4) != 0;
  const bool graph = (variant & 8) != 0;
  variant &= 3;
  const int saved_pdl = g_use_pdl;
  g_use_pdl = variant == 3 ? 1 : 0;
  auto one = [&]() {
    const uint64_t seq = ++seq_;
    const GateArgs g = make_gate(seq, 1, 0, S);
    if (variant == 0) {
      k_empty<<<S, 192, 0, s>>>();
    } else {
      int publish = variant >= 2 ? 1 : 0;
      void* args[2] = {(void*)&g, (void*)&publish};
      launch_kernel((const void*)k_gate_only, dim3(S), dim3(192), 0, s, args);
    }
  };
  for (int i = 0; i < 10; ++i) one();
  RT_CHECK(cudaStreamSynchronize(s));
  cudaGraphExec_t ge = nullptr;
  if (graph) {   // the same reps launches captured into one graph (launch cost off the host)
    cudaGraph_t gr = nullptr;
    RT_CHECK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    for (int i = 0; i < reps; ++i) one();
    RT_CHECK(cudaStreamEndCapture(s, &gr));
    RT_CHECK(cudaGraphInstantiate(&ge, gr, 0));
    cudaGraphDestroy(gr);
    RT_CHECK(cudaGraphUpload(ge, s));
    RT_CHECK(cudaStreamSynchronize(s));
  }
  RT_CHECK(cudaEventRecord(e0, s));
  const auto h0 = std::chrono::steady_clock::now();
  if (graph) {
    RT_CHECK(cudaGraphLaunch(ge, s));
  } else {
    for (int i = 0; i < reps; ++i) one();
  }
  const auto h1 = std::chrono::steady_clock::now();
  RT_CHECK(cudaEventRecord(e1, s));
  RT_CHECK(cudaEventSynchronize(e1));
  float ms = 0;
  RT_CHECK(cudaEventElapsedTime(&ms, e0, e1));
  *ns_out = host_time ? (int64_t)(std::chrono::duration<double, std::nano>(h1 - h0).count() / reps)
                      : (int64_t)(ms * 1e6 / reps);
  g_use_pdl = saved_pdl;
  if (ge) cudaGraphExecDestroy(ge);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaStreamDestroy(s);
  return true;
}

bool DeviceRT::chain_time(const std::vector<int>& hs, int lo, int hi, int graph, int reps, void* stream,
                          int64_t* device_ns, int64_t* host_ns, std::string& err) {
  cudaStream_t s = (cudaStream_t)stream;
  cudaEvent_t e0, e1;
  RT_CHECK(cudaEventCreate(&e0));
  RT_CHECK(cudaEventCreate(&e1));
  std::vector<int64_t> dv, hv;
  const int n = (int)hs.size();
  auto enqueue = [&]() -> bool {
    uint64_t prev = 0, dep = 0;
    uint32_t dep_tot = 0;
    for (int k = 0; k < n; ++k) {
      const bool stamp = k == 0 || k == n - 1;
      const uint64_t seq = alloc_seq();
      if (!launch_seq(hs[k], seq, lo, hi, s, err, stamp, prev, dep, dep_tot)) return false;
      prev = stamp ? 0 : seq;
      dep = counts(hs[k]) ? seq : 0;
      dep_tot = kernels_[hs[k]]->tiles;
    }
    return true;
  };
  for (int r = 0; r < reps + 1; ++r) {   // rep 0 is a warm-up
    RT_CHECK(cudaStreamSynchronize(s));
    cudaGraphExec_t ge = nullptr;
    if (graph) {
      cudaGraph_t g = nullptr;
      RT_CHECK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
      if (!enqueue()) { cudaStreamEndCapture(s, &g); return false; }
      RT_CHECK(cudaStreamEndCapture(s, &g));
      RT_CHECK(cudaGraphInstantiate(&ge, g, 0));
      cudaGraphDestroy(g);
      RT_CHECK(cudaGraphUpload(ge, s));
      RT_CHECK(cudaStreamSynchronize(s));
    }
    RT_CHECK(cudaEventRecord(e0, s));
    const auto h0 = std::chrono::steady_clock::now();
    if (graph) {
      RT_CHECK(cudaGraphLaunch(ge, s));
    } else if (!enqueue()) {
      return false;
    }
    const auto h1 = std::chrono::steady_clock::now();
    RT_CHECK(cudaEventRecord(e1, s));
    RT_CHECK(cudaEventSynchronize(e1));
    float ms = 0.f;
    RT_CHECK(cudaEventElapsedTime(&ms, e0, e1));
    if (ge) cudaGraphExecDestroy(ge);
    if (r > 0) {
      dv.push_back((int64_t)(ms * 1e6));
      hv.push_back((int64_t)std::chrono::duration<double, std::nano>(h1 - h0).count());
    }
  }
  std::sort(dv.begin(), dv.end());
  std::sort(hv.begin(), hv.end());
  *device_ns = dv[dv.size() / 2];
  *host_ns = hv[hv.size() / 2];
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return true;
}

bool DeviceRT::time_copy(void* dst, const void* src, size_t n, int reps, void* stream, int64_t* ns) {
  cudaStream_t st = (cudaStream_t)stream;
  cudaEvent_t a, b;
  if (cudaEventCreate(&a) != cudaSuccess || cudaEventCreate(&b) != cudaSuccess) return false;
  std::vector<float> ms;
  bool ok = true;
  for (int i = 0; i < reps + 1 && ok; ++i) {   // first copy is a warm-up
    ok = cudaEventRecord(a, st) == cudaSuccess && cudaMemcpyAsync(dst, src, n, cudaMemcpyDefault, st) == cudaSuccess &&
         cudaEventRecord(b, st) == cudaSuccess && cudaEventSynchronize(b) == cudaSuccess;
    float x = 0.f;
    if (ok && i > 0 && cudaEventElapsedTime(&x, a, b) == cudaSuccess) ms.push_back(x);
  }
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  if (!ok || ms.empty()) return false;
  std::sort(ms.begin(), ms.end());
  *ns = (int64_t)(ms[ms.size() / 2] * 1e6);
  return true;
}

bool DeviceRT::memcpy_async(void* dst, const void* src, size_t n, void* stream) {
  return cudaMemcpyAsync(dst, src, n, cudaMemcpyDefault, (cudaStream_t)stream) == cudaSuccess;
}

void DeviceRT::copy_range(uint64_t lo, uint64_t hi) {
  if (hi < lo) return;
  const uint64_t kSlotRing = ring_;
  uint64_t n = std::min<uint64_t>(hi - lo + 1, kSlotRing);
  const uint64_t s0 = lo % kSlotRing;
  const uint64_t n1 = std::min<uint64_t>(n, kSlotRing - s0);
  char* h = reinterpret_cast<char*>(stats_host_);
  const char* d = reinterpret_cast<const char*>(stats_dev_);
  cudaMemcpyAsync(h + s0 * sizeof(SlotStats), d + s0 * sizeof(SlotStats), n1 * sizeof(SlotStats),
                  cudaMemcpyDeviceToHost, (cudaStream_t)reader_);
  if (n > n1)
    cudaMemcpyAsync(h, d, (n - n1) * sizeof(SlotStats), cudaMemcpyDeviceToHost, (cudaStream_t)reader_);
}

bool DeviceRT::reader_idle() {
  if (!reader_busy_) return true;
  if (cudaEventQuery((cudaEvent_t)reader_ev_) != cudaSuccess) return false;
  reader_busy_ = false;
  return true;
}

void DeviceRT::refresh_async(uint64_t lo, uint64_t hi) {
  if (!reader_idle()) return;
  copy_range(lo, hi);
  cudaEventRecord((cudaEvent_t)reader_ev_, (cudaStream_t)reader_);
  reader_busy_ = true;
}

void DeviceRT::refresh_sync(uint64_t lo, uint64_t hi) {
  copy_range(lo, hi);
  cudaStreamSynchronize((cudaStream_t)reader_);
  reader_busy_ = false;
}

// Stats of a launch regardless of its publish state (light launches never
// publish): valid once the launch and its stream successor have finished and
// the mirror was refreshed (Engine::stop after a device sync).
void DeviceRT::peek(uint64_t seq, LaunchStats* out) {
  const volatile SlotStats* s = reinterpret_cast<const volatile SlotStats*>(stats_host_) + (seq % ring_);
  out->start_host = gt_to_host(s->start_gt);
  out->end_host = gt_to_host(s->end_gt);
  int nsm = 0;
  for (int i = 0; i < 8; ++i) nsm += __builtin_popcount(s->mask[i]);
  out->nsm = nsm;
  out->fallback = (int)(s->flags & 7u);
  for (int i = 0; i < 8; ++i) out->mask[i] = s->mask[i];
}

bool DeviceRT::poll(uint64_t seq, LaunchStats* out) {
  if (!reader_idle()) return false;  // never read the mirror while a copy is landing
  const volatile SlotStats* s = reinterpret_cast<const volatile SlotStats*>(stats_host_) + (seq % ring_);
  if (s->seq != seq) return false;
  std::atomic_thread_fence(std::memory_order_acquire);
  if (out) {
    out->start_host = gt_to_host(s->start_gt);
    out->end_host = gt_to_host(s->end_gt);
    int nsm = 0;
    for (int i = 0; i < 8; ++i) nsm += __builtin_popcount(s->mask[i]);
    out->nsm = nsm;
    out->fallback = (int)(s->flags & 7u);  // bit0: last-CTA fallback, bit1: lingering CTAs helped, bit2: software dependency timed out
    for (int i = 0; i < 8; ++i) out->mask[i] = s->mask[i];
  }
  return true;
}

void* DeviceRT::stream_create() {
  cudaStream_t s = nullptr;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  return s;
}
void DeviceRT::stream_destroy(void* s) { cudaStreamDestroy((cudaStream_t)s); }
void* DeviceRT::event_create() {
  cudaEvent_t e = nullptr;
  cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
  return e;
}
void DeviceRT::event_destroy(void* e) { cudaEventDestroy((cudaEvent_t)e); }
bool DeviceRT::event_record(void* e, void* s) { return cudaEventRecord((cudaEvent_t)e, (cudaStream_t)s) == cudaSuccess; }
bool DeviceRT::stream_wait(void* s, void* e) {
  return cudaStreamWaitEvent((cudaStream_t)s, (cudaEvent_t)e, 0) == cudaSuccess;
}
int DeviceRT::event_query(void* e) {
  const cudaError_t r = cudaEventQuery((cudaEvent_t)e);
  if (r == cudaSuccess) return 1;
  if (r == cudaErrorNotReady) return 0;
  return -1;
}
bool DeviceRT::stream_sync(void* s) { return cudaStreamSynchronize((cudaStream_t)s) == cudaSuccess; }
bool DeviceRT::device_sync() { return cudaDeviceSynchronize() == cudaSuccess; }
int64_t DeviceRT::free_bytes() {
  size_t fr = 0, tot = 0;
  return cudaMemGetInfo(&fr, &tot) == cudaSuccess ? (int64_t)fr : -1;
}

bool DeviceRT::profile(int h, int sm_count, int reps, void* stream, int64_t* ns_out, int* d_out, std::string& err) {
  cudaStream_t s = (cudaStream_t)stream;
  cudaEvent_t e0, e1;
  RT_CHECK(cudaEventCreate(&e0));
  RT_CHECK(cudaEventCreate(&e1));
  const int S = info_.sm_count;
  sm_count = std::max(1, std::min(sm_count, S));
  reps = std::max(1, reps);
  if (d_out) {
    // d (L157 "maximum active SM usage", R19): distinct SMs that processed a
    // tile in an unrestricted run -- median of 5 runs (placement varies)
    int ds[5];
    for (int r = 0; r < 5; ++r) {
      const uint64_t q = launch(h, 0, S, s, err);
      if (!q) return false;
      RT_CHECK(cudaStreamSynchronize(s));
      refresh_sync(q, q);
      LaunchStats st{};
      if (!poll(q, &st)) {
        err = "profile: launch stats missing";
        return false;
      }
      ds[r] = std::max(1, st.nsm);
    }
    std::sort(ds, ds + 5);
    *d_out = ds[2];
  }
  // timed launches use the light exit and the software dependency, as a
  // request's middle kernels do
  uint64_t prev = 0;
  const uint32_t tot = kernels_[h]->tiles;
  auto one = [&]() -> bool {
    const uint64_t q = alloc_seq();
    if (!launch_seq(h, q, 0, sm_count, s, err, false, 0, counts(h) ? prev : 0, tot)) return false;
    prev = q;
    return true;
  };
  for (int w = 0; w < 2; ++w)
    if (!one()) return false;
  float ms[3];
  for (int b = 0; b < 3; ++b) {
    RT_CHECK(cudaEventRecord(e0, s));
    for (int r = 0; r < reps; ++r)
      if (!one()) return false;
    RT_CHECK(cudaEventRecord(e1, s));
    RT_CHECK(cudaEventSynchronize(e1));
    RT_CHECK(cudaEventElapsedTime(&ms[b], e0, e1));
  }
  std::sort(ms, ms + 3);
  *ns_out = std::max<int64_t>(1, (int64_t)(ms[1] * 1.0e6 / reps + 0.5));
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return true;
}

}  // namespace bless
