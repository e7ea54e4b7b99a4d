// cuda_rt.hpp -- the CUDA side of one bl_ctx: SM probe (A1), launch-slot
// ring, gated launches (A9/A10), completion stamps (A12), offline profiler
// (A2).  Host-only declarations; implemented in cuda_rt.cu.
#pragma once
#include <cstdint>
#include <map>
#include <memory>
#include <string>
#include <vector>

#include "../../../include/bless/bless.h"
#include "kdesc.hpp"

namespace bless {

// Default launch-slot/stats ring: 2^19 records (8 MiB of slots, 32 MiB of
// stats on the device plus a 32 MiB pinned mirror); records stay readable for
// 2^18 launches, more than one bench step of any config (C4: ~31k launches).
// BLESS_STATS_RING_LOG2 (10..22) overrides it (tests).
constexpr uint64_t kSlotRingDefault = 1ull << 19;

struct LaunchStats {
  int64_t start_host, end_host;  // host clock (CLOCK_MONOTONIC ns)
  int nsm;
  int fallback;
  uint32_t mask[8];
};

class DeviceRT {
 public:
  static std::unique_ptr<DeviceRT> create(int device, void* ws, size_t ws_bytes, std::string& err);
  ~DeviceRT();

  const bl_device_info& info() const { return info_; }
  const DeviceCaps& caps() const { return caps_; }

  // Build a launch descriptor; returns its handle (index) or -1.
  int add_kernel(const bl_op& op, std::string& err);
  const KernelDesc& kernel(int h) const { return *kernels_[h]; }

  // Launch kernel h confined to logical SMs [lo, hi) on stream; returns seq (>0) or 0 on error.
  uint64_t launch(int h, int lo, int hi, void* stream, std::string& err, bool stamp = true);
  // One-CTA completion marker (stats only, no work) on stream; returns seq or 0.
  uint64_t launch_marker(void* stream, std::string& err);
  bool memcpy_async(void* dst, const void* src, size_t n, void* stream);
  // median duration (ns, CUDA events) of reps copies of n bytes on stream
  bool time_copy(void* dst, const void* src, size_t n, int reps, void* stream, int64_t* ns);
  // Diagnostics: per-launch time of back-to-back S-CTA launches.  variant 0:
  // empty kernel; 1: gate + tile queue + exit protocol; 2: 1 + host-mapped stamps.
  bool overhead(int variant, int reps, int64_t* ns_out, std::string& err);
  // Diagnostics: one request chain (kernels hs[0..n) on [lo, hi), light exits
  // for the middle kernels, PDL) launched on stream (graph = 0) or captured
  // into a CUDA graph and launched as one graph (graph = 1; capture and
  // instantiation not timed).  Median over reps of the event-timed chain
  // (device_ns) and of the host time spent enqueueing it (host_ns).
  bool chain_time(const std::vector<int>& hs, int lo, int hi, int graph, int reps, void* stream,
                  int64_t* device_ns, int64_t* host_ns, std::string& err);
  // Non-blocking: true if launch seq's stats are in the host mirror.
  bool poll(uint64_t seq, LaunchStats* out);
  void peek(uint64_t seq, LaunchStats* out);
  // Mirror the device stats of launches [lo, hi] (seq numbers) into host
  // memory: asynchronously (skipped while a previous copy is in flight) or
  // synchronously (after the launches are known complete).
  void refresh_async(uint64_t lo, uint64_t hi);
  void refresh_sync(uint64_t lo, uint64_t hi);
  uint64_t last_seq() const { return seq_; }
  // Launch-slot / stats ring: ring() records; a launch zeroes the record
  // ahead() seqs in front of it, so a record stays readable until ahead()
  // later launches have started (Engine::stop reports older light launches
  // as unknown instead of reading a reused record).
  uint64_t ring() const { return ring_; }
  uint64_t ahead() const { return ahead_; }
  // Parallel launch (Engine launcher threads): the scheduler thread allocates
  // the launch's seq; any thread may then launch it on its own stream.
  uint64_t alloc_seq() { return ++seq_; }
  // dep_seq / dep_total: the stream predecessor's seq and unit count when that
  // launch counted its units (counts() of its handle) -- this launch then
  // waits on its counter instead of griddepcontrol.wait if counts(h);
  // dep_seq = 0: hardware wait.
  bool launch_seq(int h, uint64_t seq, int lo, int hi, void* stream, std::string& err, bool stamp = true,
                  uint64_t prev_light = 0, uint64_t dep_seq = 0, uint32_t dep_total = 0);
  // Software dependency: launches of kernel h count their
  // finished units and can wait on a counting predecessor.  Opt-in
  // (BLESS_SWDEP=1): correct on B200 but not faster than griddepcontrol.wait.
  bool counts(int h) const { return swdep_ && kernels_[h]->counts_done; }
  bool launch_marker_seq(uint64_t seq, void* stream, std::string& err);

  // Streams / events (thin wrappers so the engine does not include CUDA headers).
  void* stream_create();
  void stream_destroy(void* s);
  void* event_create();
  void event_destroy(void* e);
  bool event_record(void* e, void* s);
  bool stream_wait(void* s, void* e);
  int event_query(void* e);  // 1 done, 0 pending, -1 error
  bool stream_sync(void* s);
  bool device_sync();
  bool set_device();
  int64_t free_bytes();   // cudaMemGetInfo free, -1 on error

  // Offline profiler: median over 3 batches of the per-launch mean of 'reps'
  // back-to-back launches on [0, sm_count).  d_out (if non-null): distinct SMs
  // used in one unrestricted run.
  bool profile(int h, int sm_count, int reps, void* stream, int64_t* ns_out, int* d_out, std::string& err);

  int64_t gt_to_host(int64_t gt) const { return gt - info_.clock_offset_ns; }
  bool calibrate_clock(std::string& err);
  GateArgs make_gate(uint64_t seq, uint32_t tiles, int lo, int hi, bool stamp = true, uint64_t prev_light = 0) const;

 private:
  DeviceRT() = default;
  bool probe(std::string& err);

  int device_ = 0;
  bl_device_info info_{};
  DeviceCaps caps_{};
  void* slots_ = nullptr;        // DevSlot ring (device)
  bool own_slots_ = false;
  void copy_range(uint64_t lo, uint64_t hi);
  bool reader_idle();
  void* stats_host_ = nullptr;   // pinned host mirror of the SlotStats ring
  void* stats_dev_ = nullptr;    // SlotStats ring (device memory)
  void* reader_ = nullptr;       // stream for mirror copies (copy engine)
  void* reader_ev_ = nullptr;
  bool reader_busy_ = false;
  uint8_t* lid_map_dev_ = nullptr;
  bool identity_map_ = true;
  uint64_t seq_ = 0;
  uint32_t linger_ns_ = 30000;   // GateArgs::linger_ns (BLESS_LINGER_NS)
  bool swdep_ = false;           // BLESS_SWDEP=1 enables (measured no gain on B200)
  uint64_t ring_ = kSlotRingDefault;
  uint64_t ahead_ = kSlotRingDefault / 2;
  std::vector<std::unique_ptr<KernelDesc>> kernels_;
  bool autotune_ = true;          // BLESS_TC_AUTOTUNE=0 keeps the builder's heuristic
  void* tune_stream_ = nullptr;
  bool autotune_tc(const bl_op& op, std::unique_ptr<KernelDesc>& best, std::string& err);
  std::string tc_signature(const bl_op& op) const;
  std::map<std::string, TcChoice> tune_cache_;   // BLESS_TC_TUNE_FILE
  std::string tune_file_;
};

}  // namespace bless
