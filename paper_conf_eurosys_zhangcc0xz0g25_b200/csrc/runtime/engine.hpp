// engine.hpp -- one bl_ctx: tenants, request table, scheduler/launch thread,
// policies (BLESS + in-run baselines), logs.  Host C++17; device work goes
// through DeviceRT (null for BL_DEVICE_NONE contexts, which run the same
// scheduler on the virtual clock without CUDA).
#pragma once
#include <atomic>
#include <deque>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "../../../include/bless/bless.h"
#include "../sched/sched.hpp"

namespace bless {

class DeviceRT;

struct Req {
  std::atomic<int> published{0};
  std::atomic<int> done{0};
  int tenant = 0;
  int64_t arrival = 0;       // as submitted
  int64_t arrival_host = 0;  // latency origin (host clock; model time without a device)
  int64_t start = 0, finish = 0;
};

struct TenantRT {
  std::string name;
  int64_t ppm = 0;
  std::vector<int> handles;  // DeviceRT kernel handles
  void* stream = nullptr;
  bool own_stream = false;
  int lo = 0, hi = 0;        // static (ISO/STATIC) range
  std::vector<void*> events; // ring for squad barriers
  size_t ev_next = 0;
  // per-request host I/O (bl_set_tenant_io)
  const void* host_in = nullptr;
  void* dev_in = nullptr;
  size_t in_bytes = 0;
  const void* dev_out = nullptr;
  void* host_out = nullptr;
  size_t out_bytes = 0;
  uint64_t prev_light = 0;   // last launch on the stream if it used the light exit (owned by its launcher)
  uint64_t dep_seq = 0;      // last launch on the stream if it counted its units (software dependency), else 0
  uint32_t dep_tot = 0;      //   and its unit count
};

// Parallel launch path.  Host launch calls cost ~3 us each on the B200 boxes
// (kprobe: cudaLaunchKernelExC ~ 3.0-3.4 us per call), about the device time
// of a batch-1 kernel, so one host thread launching every tenant's kernels
// serialises co-running tenants on the CPU.  Each tenant stream gets its own
// launcher thread; the scheduler thread decides, allocates the launches' seqs
// and logs them, and hands a LaunchJob to the tenant's launcher.
struct LaunchItem {
  enum Kind : uint8_t { KERNEL = 0, H2D = 1, D2H = 2, MARKER = 3 };
  uint8_t kind = KERNEL;
  uint8_t stamp = 1;    // full exit protocol (host observes completion); 0 = light exit
  int handle = -1;
  uint64_t seq = 0;
  int lo = 0, hi = 0;
};

struct LaunchJob {
  uint64_t squad = 0;             // squad id (0: none -- baseline policies)
  uint64_t wait_squad = 0;        // squad barrier: every launcher in wait_parts
  std::vector<int> wait_parts;    //   must have recorded squad wait_squad first
  std::vector<uint64_t> wait_sq;  //   (per part when non-empty: barrier = 1),
  std::vector<void*> wait_events; //   then its stream waits on wait_events
  std::vector<LaunchItem> items;
  void* record_event = nullptr;   // recorded after the items (squad barrier)
};

struct Launcher {
  std::thread th;
  std::mutex mu;
  std::deque<LaunchJob> q;
  std::atomic<size_t> queued{0};
  std::atomic<bool> quit{false};
  std::atomic<uint64_t> recorded{0};   // last squad whose barrier event this launcher recorded
};

struct PendingLaunch {
  uint64_t seq;
  size_t log_idx;
  int64_t req;   // request whose first/last kernel this is (-1 otherwise)
  int kernel;
  int last;      // 1 if this is the request's last kernel
};

class Engine {
 public:
  Engine(int device, const bl_params& p);
  ~Engine();
  bl_status init(void* ws, size_t ws_bytes, std::string& err);

  bl_status register_tenant(double quota, const char* name, int* out, std::string& err);
  bl_status set_slo(int t, int64_t slo_ns, std::string& err);
  bl_status set_stream(int t, void* s, std::string& err);
  bl_status append_kernel(int t, const bl_op* op, int* out, std::string& err);
  bl_status run_kernel(int t, int k, int lo, int hi, std::string& err);
  bl_status kernel_info(int t, int k, bl_kernel_info* out, std::string& err);
  bl_status debug_overhead(int variant, int reps, int64_t* ns, std::string& err);
  bl_status debug_chain(int t, int lo, int hi, int graph, int reps, int64_t* dev_ns, int64_t* host_ns, std::string& err);
  bl_status set_io(int t, const void* hin, void* din, size_t inb, const void* dout, void* hout, size_t outb,
                   std::string& err);
  bl_status profile_kernel(int t, int k, int sm_count, int reps, int64_t* ns, int* d, std::string& err);
  bl_status profile_tenant(int t, int reps, std::string& err);
  bl_status set_profile_row(int t, int k, const int64_t* tns, int d, std::string& err);
  bl_status get_profile_row(int t, int k, int64_t* tns, int* d, std::string& err);
  bl_status save_profile(const char* path, std::string& err);
  bl_status load_profile(const char* path, std::string& err);
  bl_status tenant_info(int t, int* qsms, int* m, int64_t* T, std::string& err);
  bl_status device_info(bl_device_info* out, std::string& err);

  bl_status start(std::string& err);
  bl_status submit(int t, int64_t arrival, uint64_t* out, std::string& err);
  bl_status poll(uint64_t req, bl_req_info* out, std::string& err);
  bl_status drain(int64_t timeout_ns, std::string& err);
  bl_status stop(std::string& err);
  bl_status reset(const bl_params* p, std::string& err);
  bl_status decisions(size_t first, bl_decision* buf, size_t cap, size_t* n);
  bl_status launches(size_t first, bl_launch_rec* buf, size_t cap, size_t* n);
  bl_status decide_pure(int64_t now, int n, const int32_t* ten, const int64_t* arr, const int32_t* nxt,
                        bl_decision* out, std::string& err);
  bl_status temporal_log(size_t first, bl_temporal_rec* buf, size_t cap, size_t* n);
  bl_status time_decide(const bl_decision* recs, size_t n, int reps, int64_t* total_ns, int64_t* picks,
                        std::string& err);
  bool virtual_clock() const { return prm_.clock == BL_CLOCK_VIRTUAL; }
  bl_status deployment_check(const int64_t* mem, int64_t free_b, int32_t span, int32_t* ok, int32_t* why,
                             std::string& err);
  bl_status predict(int n, const int32_t* ten, const int32_t* ker, const int32_t* p, int64_t* out, std::string& err);
  bl_status run_squad(int n, const int32_t* ten, const int32_t* ker, const int16_t* lo, const int16_t* hi, int reps,
                      int64_t* makespan, int64_t* kernel_ns, std::string& err);

 private:
  void thread_main();
  void loop_bless();
  void loop_at_arrival(bool unbound);
  void loop_temporal();
  void scan_submissions();
  void harvest();
  void retire_inflight();
  void launch_squad(const Decision& d, const std::vector<int64_t>& act_req, const std::vector<int>& act_next,
                    bool join_solo = false);
  uint64_t launch_one(int t, int k, int lo, int hi, void* stream, int64_t req, bool last, bool stamp = true);
  // parallel launch path
  bool prepare_one(int t, int k, int lo, int hi, int64_t req, bool last, std::vector<LaunchItem>& items,
                   bool stamp = true);
  bool exec_items(int t, const std::vector<LaunchItem>& items, void* stream, std::string& err);
  void push_job(int t, LaunchJob&& job);
  void launcher_main(int t);
  void start_launchers();
  void stop_launchers();
  bool use_launchers() const { return rt_ && prm_.policy != BL_POLICY_TEMPORAL; }
  void log_decision(const Decision& d);
  void fail(const std::string& msg);
  int nten() const { return (int)ten_.size(); }
  int S() const { return prof_.S; }

  int device_;
  bl_params prm_;
  std::unique_ptr<DeviceRT> rt_;
  Profile prof_;
  Profile prof_full_;        // the whole-GPU profile while a run is restricted by sm_limit
  bool limited_ = false;
  std::vector<TenantRT> ten_;
  double quota_sum_ = 0;

  // request table
  std::unique_ptr<Req[]> reqs_;
  int64_t cap_ = 0;
  std::atomic<uint64_t> next_id_{0};
  std::atomic<uint64_t> n_done_{0};
  std::vector<int64_t> last_submit_arrival_;

  // thread
  std::thread th_;
  std::atomic<bool> stop_{false};
  std::atomic<bool> started_{false};
  std::atomic<bool> failed_{false};
  std::string fail_msg_;
  int64_t t0_ = 0;

  // scheduler-thread state
  uint64_t scan_ = 0;
  std::vector<std::deque<uint64_t>> fifo_;
  DecideScratch scratch_;
  Decision dec_;
  std::vector<PendingLaunch> pending_;
  uint64_t run_first_seq_ = 1;
  int64_t last_refresh_ns_ = 0;
  bool harvest_all_ = false;
  struct Inflight {
    std::vector<void*> events;
    std::vector<int> parts;
    uint64_t squad = 0;
    bool solo_nsp = false;   // one participant on [0, S) (R38)
  };
  // R38 (bl_params.barrier bit 1): the tenant whose solo NSP squads are all
  // that is in flight, or -1
  int solo_inflight_tenant() const;
  std::vector<std::unique_ptr<Launcher>> launchers_;
  uint64_t squad_id_ = 0;
  bool par_launch_ = true;        // per-tenant launcher threads (BLESS_LAUNCH_THREADS=0 disables)
  std::vector<int> prev_parts_;
  uint64_t prev_squad_ = 0;
  std::deque<Inflight> inflight_;
  std::vector<void*> prev_events_;
  // SM-range barrier (bl_params.barrier = 1, reading R37): per tenant, its
  // latest chain's end event, squad id and the logical SMs its kernels used
  struct LastChain {
    void* ev = nullptr;
    uint64_t squad = 0;
    uint64_t mask[3] = {0, 0, 0};
  };
  std::vector<LastChain> last_chain_;
  void* temporal_stream_ = nullptr;

  // logs
  std::mutex log_mu_;
  std::vector<bl_decision> dlog_;
  std::vector<bl_launch_rec> llog_;
  std::vector<bl_temporal_rec> tlog_;
};

}  // namespace bless
