// engine.cpp -- see engine.hpp.  Paper citations are PAPER.md lines; readings
// R<n> are DESIGN.md §3.
#include "engine.hpp"

#include <algorithm>
#include <array>
#include <chrono>
#include <climits>
#include <cmath>
#include <cstdlib>
#include <cstring>

#include "cuda_rt.hpp"

namespace bless {

static int64_t now_ns() {
  return std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

static inline void cpu_relax() {
#if defined(__x86_64__)
  __builtin_ia32_pause();
#endif
}

Engine::Engine(int device, const bl_params& p) : device_(device), prm_(p) {}

Engine::~Engine() {
  std::string e;
  stop(e);
  if (rt_) {
    rt_->set_device();
    rt_->device_sync();
    for (auto& t : ten_) {
      for (void* ev : t.events) rt_->event_destroy(ev);
      if (t.own_stream && t.stream) rt_->stream_destroy(t.stream);
    }
    if (temporal_stream_) rt_->stream_destroy(temporal_stream_);
  }
}

bl_status Engine::init(void* ws, size_t ws_bytes, std::string& err) {
  if (prm_.sm_unit < 1 || prm_.squad_max < 1 || prm_.squad_max > BL_MAX_SQUAD || prm_.split_pct < 0 ||
      prm_.ablate < 0 || prm_.ablate > 3 || prm_.squad_max_solo < 0 || prm_.squad_max_solo > BL_MAX_SQUAD ||
      prm_.split_pct > 100 || prm_.max_requests < 1 || prm_.barrier < 0 || prm_.barrier > 3) {
    err = "invalid bl_params";
    return BL_E_INVALID;
  }
  if (device_ != BL_DEVICE_NONE) {
    rt_ = DeviceRT::create(device_, ws, ws_bytes, err);
    if (!rt_) return BL_E_CUDA;
    prof_.S = rt_->info().sm_count;
  }
  prof_.g = prm_.sm_unit;
  cap_ = prm_.max_requests;
  reqs_.reset(new (std::nothrow) Req[cap_]);
  if (!reqs_) { err = "request table alloc"; return BL_E_OOM; }
  return BL_OK;
}

void Engine::fail(const std::string& msg) {
  if (!failed_.exchange(true)) fail_msg_ = msg;
  stop_ = true;
}

// ------------------------------------------------------------------ setup
bl_status Engine::register_tenant(double quota, const char* name, int* out, std::string& err) {
  if (started_) { err = "register after bl_start"; return BL_E_STATE; }
  if (!(quota > 0.0) || quota > 1.0) { err = "quota must be in (0, 1]"; return BL_E_QUOTA; }
  if (quota_sum_ + quota > 1.0 + 1e-9) { err = "sum of quotas exceeds 1"; return BL_E_QUOTA; }
  if (nten() >= BL_MAX_TENANTS) { err = "too many tenants"; return BL_E_FULL; }
  TenantRT t;
  t.name = name && *name ? name : ("tenant" + std::to_string(nten()));
  for (char& c : t.name)
    if (c == ' ' || c == '\t' || c == '\n') c = '_';
  t.ppm = std::llround(quota * 1e6);
  if (rt_) {
    rt_->set_device();
    t.stream = rt_->stream_create();
    t.own_stream = true;
    for (int i = 0; i < 64; ++i) t.events.push_back(rt_->event_create());
  }
  quota_sum_ += quota;
  TenantProfile tp;
  tp.name = t.name;
  tp.quota_ppm = t.ppm;
  prof_.ten.push_back(tp);
  ten_.push_back(std::move(t));
  if (out) *out = nten() - 1;
  return BL_OK;
}

bl_status Engine::set_slo(int t, int64_t slo_ns, std::string& err) {
  if (t < 0 || t >= nten() || slo_ns < 0) { err = "bad tenant/slo"; return BL_E_INVALID; }
  if (started_) { err = "set_slo after bl_start"; return BL_E_STATE; }
  prof_.ten[t].slo_ns = slo_ns;
  prof_.derive();
  return BL_OK;
}

bl_status Engine::set_stream(int t, void* s, std::string& err) {
  if (t < 0 || t >= nten() || !s) { err = "bad tenant/stream"; return BL_E_INVALID; }
  if (started_) { err = "set_stream after bl_start"; return BL_E_STATE; }
  if (!rt_) { err = "no device"; return BL_E_STATE; }
  if (ten_[t].own_stream) rt_->stream_destroy(ten_[t].stream);
  ten_[t].stream = s;
  ten_[t].own_stream = false;
  return BL_OK;
}

bl_status Engine::append_kernel(int t, const bl_op* op, int* out, std::string& err) {
  if (t < 0 || t >= nten() || !op) { err = "bad tenant/op"; return BL_E_INVALID; }
  if (started_) { err = "append after bl_start"; return BL_E_STATE; }
  KernelProfile kp;
  if (rt_) {
    rt_->set_device();
    const int h = rt_->add_kernel(*op, err);
    if (h < 0) return BL_E_INVALID;
    ten_[t].handles.push_back(h);
    kp.name = std::string(rt_->kernel(h).family) + "_" + std::to_string(prof_.ten[t].k.size());
  } else {
    if (op->kind != BL_OP_VIRTUAL) { err = "device-less ctx accepts BL_OP_VIRTUAL only"; return BL_E_INVALID; }
    ten_[t].handles.push_back(-1);
    kp.name = "virtual_" + std::to_string(prof_.ten[t].k.size());
  }
  prof_.ten[t].k.push_back(kp);
  if (out) *out = (int)prof_.ten[t].k.size() - 1;
  return BL_OK;
}

bl_status Engine::run_kernel(int t, int k, int lo, int hi, std::string& err) {
  if (!rt_) { err = "no device"; return BL_E_STATE; }
  if (t < 0 || t >= nten() || k < 0 || k >= (int)ten_[t].handles.size()) { err = "bad index"; return BL_E_INVALID; }
  if (started_) { err = "run_kernel while running"; return BL_E_STATE; }
  rt_->set_device();
  lo = std::max(0, lo);
  hi = std::min(S(), hi);
  if (lo >= hi) { err = "empty SM range"; return BL_E_INVALID; }
  const uint64_t seq = rt_->launch(ten_[t].handles[k], lo, hi, ten_[t].stream, err);
  if (!seq) return BL_E_CUDA;
  if (!rt_->stream_sync(ten_[t].stream)) { err = "stream sync failed (kernel fault?)"; return BL_E_CUDA; }
  return BL_OK;
}

bl_status Engine::set_io(int t, const void* hin, void* din, size_t inb, const void* dout, void* hout, size_t outb,
                         std::string& err) {
  if (!rt_) { err = "no device"; return BL_E_STATE; }
  if (t < 0 || t >= nten()) { err = "bad tenant"; return BL_E_INVALID; }
  if (started_) { err = "set_io after bl_start"; return BL_E_STATE; }
  if ((inb && (!hin || !din)) || (outb && (!dout || !hout))) { err = "null io buffer"; return BL_E_INVALID; }
  TenantRT& tr = ten_[t];
  tr.host_in = hin;
  tr.dev_in = din;
  tr.in_bytes = inb;
  tr.dev_out = dout;
  tr.host_out = hout;
  tr.out_bytes = outb;
  // profile the memory-management kernels for the predictors (L229, R31)
  rt_->set_device();
  TenantProfile& tp = prof_.ten[t];
  tp.io_in = tp.io_out = 0;
  if (inb && !rt_->time_copy(din, hin, inb, 5, tr.stream, &tp.io_in)) { err = "H2D copy failed"; return BL_E_CUDA; }
  if (outb && !rt_->time_copy(hout, dout, outb, 5, tr.stream, &tp.io_out)) { err = "D2H copy failed"; return BL_E_CUDA; }
  prof_.derive();
  return BL_OK;
}

bl_status Engine::debug_overhead(int variant, int reps, int64_t* ns, std::string& err) {
  if (!rt_) { err = "no device"; return BL_E_STATE; }
  if (started_) { err = "diagnostics while running"; return BL_E_STATE; }
  if (!ns || variant < 0 || variant > 15 || reps < 1) { err = "bad args"; return BL_E_INVALID; }
  rt_->set_device();
  return rt_->overhead(variant, reps, ns, err) ? BL_OK : BL_E_CUDA;
}

bl_status Engine::debug_chain(int t, int lo, int hi, int graph, int reps, int64_t* dev_ns, int64_t* host_ns,
                              std::string& err) {
  if (!rt_) { err = "no device"; return BL_E_STATE; }
  if (started_) { err = "diagnostics while running"; return BL_E_STATE; }
  if (t < 0 || t >= nten() || lo < 0 || hi > S() || lo >= hi || reps < 1 || !dev_ns || !host_ns) {
    err = "bad args";
    return BL_E_INVALID;
  }
  rt_->set_device();
  return rt_->chain_time(ten_[t].handles, lo, hi, graph, reps, ten_[t].stream, dev_ns, host_ns, err) ? BL_OK
                                                                                                       : BL_E_CUDA;
}

bl_status Engine::kernel_info(int t, int k, bl_kernel_info* out, std::string& err) {
  if (!rt_) { err = "no device"; return BL_E_STATE; }
  if (t < 0 || t >= nten() || k < 0 || k >= (int)ten_[t].handles.size() || !out) { err = "bad index"; return BL_E_INVALID; }
  const KernelDesc& d = rt_->kernel(ten_[t].handles[k]);
  std::memset(out, 0, sizeof(*out));
  std::strncpy(out->family, d.family, sizeof(out->family) - 1);
  out->tiles = (int32_t)d.tiles;
  out->grid = d.grid;
  out->block = d.block;
  out->smem = d.smem;
  out->flops = d.flops;
  out->bytes = d.bytes;
  return BL_OK;
}

bl_status Engine::profile_kernel(int t, int k, int sm_count, int reps, int64_t* ns, int* d, std::string& err) {
  if (!rt_) { err = "no device"; return BL_E_STATE; }
  if (started_) { err = "profile while running"; return BL_E_STATE; }
  if (t < 0 || t >= nten() || k < 0 || k >= (int)ten_[t].handles.size() || !ns) { err = "bad index"; return BL_E_INVALID; }
  rt_->set_device();
  if (!rt_->profile(ten_[t].handles[k], sm_count, reps, ten_[t].stream, ns, d, err)) return BL_E_CUDA;
  return BL_OK;
}

bl_status Engine::profile_tenant(int t, int reps, std::string& err) {
  if (!rt_) { err = "no device"; return BL_E_STATE; }
  if (t < 0 || t >= nten()) { err = "bad tenant"; return BL_E_INVALID; }
  const int Sx = S();
  for (size_t k = 0; k < ten_[t].handles.size(); ++k) {
    KernelProfile& kp = prof_.ten[t].k[k];
    kp.t.assign(Sx, 0);
    int d = 0;
    int64_t ns = 0;
    bl_status st = profile_kernel(t, (int)k, Sx, reps, &ns, &d, err);
    if (st != BL_OK) return st;
    kp.d = d;
    kp.t[Sx - 1] = ns;
    for (int s = 1; s < Sx; ++s) {
      st = profile_kernel(t, (int)k, s, reps, &kp.t[s - 1], nullptr, err);
      if (st != BL_OK) return st;
    }
  }
  prof_.derive();
  // tau[n%][k] and T[n%] (L157, reading R35): "the duration from the
  // beginning of the application to the end of k", measured along isolated
  // runs of the whole request on the tenant's quota SMs, launched exactly as
  // the engine launches a request (programmatic dependent launch, light exits
  // for the middle kernels); element-wise median over the runs
  // Opt-in (BLESS_MEASURED_TAU=1): on B200 the measured chains are shorter
  // than the per-kernel prefix sums (R50 at 99 SMs: 0.44 vs 0.51 ms) and the
  // C2 bench got 5% slower with them (profiles/round2/bench/), so the default
  // keeps the round-1 prefix sums.
  TenantProfile& tp = prof_.ten[t];
  const int q = tp.quota_sms;
  const int m = (int)ten_[t].handles.size();
  const char* mt = std::getenv("BLESS_MEASURED_TAU");
  if (mt && std::atoi(mt) != 0 && q >= 1 && m > 0) {
    rt_->set_device();
    const int runs = std::max(3, reps);
    std::vector<std::vector<int64_t>> tau(m);
    for (int r = 0; r < runs + 1; ++r) {   // run 0 warms up
      if (!rt_->device_sync()) { err = "device error before the tau run"; return BL_E_CUDA; }
      std::vector<uint64_t> seqs(m);
      uint64_t prev_light = 0, dep = 0;
      uint32_t dep_tot = 0;
      for (int k = 0; k < m; ++k) {
        const bool stamp = k == 0 || k == m - 1;
        const int h = ten_[t].handles[k];
        seqs[k] = rt_->alloc_seq();
        if (!rt_->launch_seq(h, seqs[k], 0, q, ten_[t].stream, err, stamp, prev_light, dep, dep_tot))
          return BL_E_CUDA;
        prev_light = stamp ? 0 : seqs[k];
        dep = rt_->counts(h) ? seqs[k] : 0;
        dep_tot = rt_->kernel(h).tiles;
      }
      if (!rt_->device_sync()) { err = "device error in the tau run"; return BL_E_CUDA; }
      if (r == 0) continue;
      rt_->refresh_sync(seqs.front(), seqs.back());
      LaunchStats s0{};
      rt_->peek(seqs[0], &s0);
      for (int k = 0; k < m; ++k) {
        LaunchStats st{};
        rt_->peek(seqs[k], &st);
        tau[k].push_back(std::max<int64_t>(1, st.end_host - s0.start_host));
      }
    }
    tp.tau_meas.assign(m, 0);
    for (int k = 0; k < m; ++k) {
      std::sort(tau[k].begin(), tau[k].end());
      tp.tau_meas[k] = tau[k][tau[k].size() / 2];
      if (k && tp.tau_meas[k] < tp.tau_meas[k - 1]) tp.tau_meas[k] = tp.tau_meas[k - 1];   // medians of a monotone chain
    }
    tp.tau_sms = q;
    prof_.derive();
  }
  return BL_OK;
}

bl_status Engine::set_profile_row(int t, int k, const int64_t* tns, int d, std::string& err) {
  if (t < 0 || t >= nten() || k < 0 || k >= (int)prof_.ten[t].k.size() || !tns || d < 1 || d > S()) {
    err = "bad profile row";
    return BL_E_INVALID;
  }
  if (started_) { err = "profile change while running"; return BL_E_STATE; }
  prof_.ten[t].k[k].t.assign(tns, tns + S());
  prof_.ten[t].k[k].d = d;
  prof_.derive();
  return BL_OK;
}

bl_status Engine::get_profile_row(int t, int k, int64_t* tns, int* d, std::string& err) {
  if (t < 0 || t >= nten() || k < 0 || k >= (int)prof_.ten[t].k.size()) { err = "bad index"; return BL_E_INVALID; }
  const auto& kp = prof_.ten[t].k[k];
  if ((int)kp.t.size() != S()) { err = "kernel not profiled"; return BL_E_STATE; }
  if (tns) std::memcpy(tns, kp.t.data(), sizeof(int64_t) * S());
  if (d) *d = kp.d;
  return BL_OK;
}

bl_status Engine::save_profile(const char* path, std::string& err) {
  if (!path) { err = "null path"; return BL_E_INVALID; }
  if (!prof_.complete()) { err = "profile incomplete"; return BL_E_STATE; }
  return save_profile_text(path, prof_, err) ? BL_OK : BL_E_INVALID;
}

bl_status Engine::load_profile(const char* path, std::string& err) {
  if (!path) { err = "null path"; return BL_E_INVALID; }
  if (started_) { err = "load after bl_start"; return BL_E_STATE; }
  Profile p;
  if (!load_profile_text(path, p, err)) return BL_E_NOTFOUND;
  if (!rt_ && nten() == 0) {
    // device-less ctx: adopt the whole description
    prm_.sm_unit = p.g;
    for (auto& tn : p.ten) {
      int id = 0;
      bl_status st = register_tenant((double)tn.quota_ppm / 1e6, tn.name.c_str(), &id, err);
      if (st != BL_OK) return st;
      ten_[id].ppm = tn.quota_ppm;  // exact
      for (size_t k = 0; k < tn.k.size(); ++k) ten_[id].handles.push_back(-1);
    }
    prof_ = p;
    prof_.derive();
    return BL_OK;
  }
  if (p.S != S() || (int)p.ten.size() != nten()) { err = "profile does not match this ctx (S or tenants)"; return BL_E_INVALID; }
  for (int j = 0; j < nten(); ++j) {
    if (p.ten[j].k.size() != prof_.ten[j].k.size() || p.ten[j].quota_ppm != prof_.ten[j].quota_ppm) {
      err = "profile does not match tenant " + std::to_string(j);
      return BL_E_INVALID;
    }
    if (p.ten[j].slo_ns > 0) prof_.ten[j].slo_ns = p.ten[j].slo_ns;
    if (p.ten[j].io_in > 0 || p.ten[j].io_out > 0) {
      prof_.ten[j].io_in = p.ten[j].io_in;
      prof_.ten[j].io_out = p.ten[j].io_out;
    }
    prof_.ten[j].tau_sms = p.ten[j].tau_sms;
    prof_.ten[j].tau_meas = p.ten[j].tau_meas;
    for (size_t k = 0; k < p.ten[j].k.size(); ++k) {
      prof_.ten[j].k[k].t = p.ten[j].k[k].t;
      prof_.ten[j].k[k].d = p.ten[j].k[k].d;
    }
  }
  prof_.g = p.g;
  prm_.sm_unit = p.g;
  prof_.derive();
  return BL_OK;
}

bl_status Engine::tenant_info(int t, int* qsms, int* m, int64_t* T, std::string& err) {
  if (t < 0 || t >= nten()) { err = "bad tenant"; return BL_E_INVALID; }
  prof_.derive();
  if (qsms) *qsms = prof_.ten[t].quota_sms;
  if (m) *m = (int)prof_.ten[t].k.size();
  if (T) *T = prof_.ten[t].T;
  return BL_OK;
}

bl_status Engine::device_info(bl_device_info* out, std::string& err) {
  if (!out) { err = "null"; return BL_E_INVALID; }
  if (!rt_) { err = "no device"; return BL_E_STATE; }
  *out = rt_->info();
  return BL_OK;
}

// ------------------------------------------------------------------ runtime
bl_status Engine::start(std::string& err) {
  if (started_) { err = "already started"; return BL_E_STATE; }
  if (nten() == 0) { err = "no tenants"; return BL_E_STATE; }
  if (!prof_.complete()) { err = "submit/start before a complete profile (PAPER.md L155: no profile, no BLESS)"; return BL_E_STATE; }
  prof_.g = prm_.sm_unit;
  if (prm_.sm_limit) {
    // f4 SM-count sweep (L420): the whole system runs on logical SMs
    // [0, sm_limit) -- profile columns 1..sm_limit, d capped, N = sm_limit/g
    if (prm_.sm_limit < prm_.sm_unit || prm_.sm_limit > prof_.S) { err = "sm_limit outside [g, S]"; return BL_E_INVALID; }
    prof_full_ = prof_;
    limited_ = true;
    prof_.S = prm_.sm_limit;
    for (auto& tn : prof_.ten)
      for (auto& k : tn.k) {
        k.t.resize(prof_.S);
        k.d = std::min(k.d, prof_.S);
      }
  }
  prof_.derive();
  if (prof_.N < 1) { err = "sm_unit larger than S"; return BL_E_INVALID; }
  int lo = 0;
  for (int j = 0; j < nten(); ++j) {
    if (prof_.ten[j].quota_sms < 1) { err = "tenant " + std::to_string(j) + " gets 0 SMs"; return BL_E_QUOTA; }
    if (prof_.ten[j].k.empty()) { err = "tenant without kernels"; return BL_E_STATE; }
    ten_[j].lo = lo;
    ten_[j].hi = lo + prof_.ten[j].quota_sms;
    lo = ten_[j].hi;
    ten_[j].prev_light = 0;   // no stream predecessor from before this run (its ring records may be reused)
    ten_[j].dep_seq = 0;
  }
  if (!rt_ && prm_.policy != BL_POLICY_BLESS) { err = "device-less ctx runs the BLESS policy only"; return BL_E_STATE; }
  if (!rt_ && prm_.clock != BL_CLOCK_VIRTUAL) { err = "device-less ctx needs the VIRTUAL clock"; return BL_E_STATE; }
  if (rt_) {
    rt_->set_device();
    if (!temporal_stream_) temporal_stream_ = rt_->stream_create();
    rt_->calibrate_clock(err);
  }
  fifo_.assign(nten(), {});
  scan_ = 0;
  pending_.clear();
  if (rt_) run_first_seq_ = rt_->last_seq() + 1;
  inflight_.clear();
  prev_events_.clear();
  prev_parts_.clear();
  prev_squad_ = 0;
  last_chain_.assign(nten(), LastChain{});
  stop_ = false;
  failed_ = false;
  t0_ = now_ns() + 1000000;  // VIRTUAL on a device: wall anchor of trace time 0
  started_ = true;
  par_launch_ = true;
  if (const char* e = std::getenv("BLESS_LAUNCH_THREADS")) par_launch_ = std::atoi(e) != 0;
  start_launchers();
  th_ = std::thread([this] { thread_main(); });
  return BL_OK;
}

bl_status Engine::submit(int t, int64_t arrival, uint64_t* out, std::string& err) {
  if (t < 0 || t >= nten()) { err = "bad tenant"; return BL_E_INVALID; }
  if (prm_.clock == BL_CLOCK_VIRTUAL && started_) { err = "VIRTUAL clock: submit the whole trace before bl_start"; return BL_E_STATE; }
  if (!prof_.complete()) { err = "submit before a complete profile"; return BL_E_STATE; }
  if (prm_.clock == BL_CLOCK_VIRTUAL) {
    if ((int)last_submit_arrival_.size() < nten()) last_submit_arrival_.resize(nten(), INT64_MIN);
    if (arrival < last_submit_arrival_[t]) { err = "VIRTUAL: arrivals must be non-decreasing per tenant"; return BL_E_INVALID; }
    last_submit_arrival_[t] = arrival;
  }
  const uint64_t id = next_id_.fetch_add(1);
  if ((int64_t)id >= cap_) { err = "request table full"; return BL_E_FULL; }
  Req& r = reqs_[id];
  r.tenant = t;
  r.arrival = arrival;
  r.arrival_host = arrival;
  r.start = r.finish = 0;
  r.done.store(0, std::memory_order_relaxed);
  r.published.store(1, std::memory_order_release);
  if (out) *out = id;
  return BL_OK;
}

bl_status Engine::poll(uint64_t id, bl_req_info* out, std::string& err) {
  if (id >= next_id_.load() || (int64_t)id >= cap_) { err = "unknown request"; return BL_E_NOTFOUND; }
  Req& r = reqs_[id];
  if (out) {
    out->req = id;
    out->tenant = r.tenant;
    out->arrival_ns = r.arrival_host;
  }
  if (!r.done.load(std::memory_order_acquire)) {
    if (out) out->status = BL_PENDING;
    if (failed_) { err = "engine failed: " + fail_msg_; return BL_E_CUDA; }
    return BL_PENDING;
  }
  if (out) {
    out->status = BL_OK;
    out->start_ns = r.start;
    out->finish_ns = r.finish;
  }
  return BL_OK;
}

bl_status Engine::drain(int64_t timeout_ns, std::string& err) {
  const int64_t deadline = now_ns() + timeout_ns;
  while (n_done_.load() < next_id_.load()) {
    if (failed_) { err = "engine failed: " + fail_msg_; return BL_E_CUDA; }
    if (!started_) { err = "not started"; return BL_E_STATE; }
    if (timeout_ns >= 0 && now_ns() > deadline) { err = "drain timeout"; return BL_E_TIMEOUT; }
    std::this_thread::sleep_for(std::chrono::microseconds(50));
  }
  return BL_OK;
}

bl_status Engine::stop(std::string& err) {
  stop_ = true;
  if (th_.joinable()) th_.join();
  stop_launchers();
  if (rt_ && started_) {
    rt_->set_device();
    if (!rt_->device_sync()) { err = "device error at stop"; started_ = false; return BL_E_CUDA; }
    // every launch of the run has finished: mirror the whole stats range once
    // (includes the SM masks) and complete the logs
    // Records older than ahead() launches have been zeroed for reuse by later
    // launches: only the last ahead() seqs are read back; an older light
    // launch (never published, so not harvested during the run) is reported
    // as unknown (nsm = -1, no times) instead of from a reused record.
    const uint64_t hi = rt_->last_seq();
    const uint64_t win = rt_->ahead();
    const uint64_t lo = hi >= run_first_seq_ ? std::max<uint64_t>(run_first_seq_, hi > win ? hi - win + 1 : 1) : hi + 1;
    rt_->refresh_sync(lo, hi);
    harvest_all_ = true;
    harvest();
    harvest_all_ = false;
    std::lock_guard<std::mutex> lk(log_mu_);
    for (bl_launch_rec& r : llog_) {
      LaunchStats st;
      if (r.seq < lo && r.end_ns == 0) {
        r.nsm = -1;
        r.start_ns = 0;
      } else if (r.seq >= lo && r.seq <= hi) {
        rt_->peek(r.seq, &st);   // light launches never publish their seq
        r.start_ns = st.start_host;
        r.end_ns = st.end_host;
        r.nsm = st.nsm;
        r.fallback = st.fallback;
        for (int i = 0; i < 8; ++i) r.sm_mask[i] = st.mask[i];
      }
    }
  }
  started_ = false;
  if (limited_) {   // back to the whole-GPU profile
    prof_ = prof_full_;
    limited_ = false;
  }
  if (failed_) { err = fail_msg_; return BL_E_CUDA; }
  return BL_OK;
}

bl_status Engine::deployment_check(const int64_t* mem, int64_t free_b, int32_t span, int32_t* ok, int32_t* why,
                                   std::string& err) {
  if (!mem || !ok || span < 1) { err = "bad args"; return BL_E_INVALID; }
  if (!prof_.complete()) { err = "profile incomplete"; return BL_E_STATE; }
  if (free_b <= 0) {
    if (!rt_) { err = "no device to query free memory"; return BL_E_STATE; }
    rt_->set_device();
    free_b = rt_->free_bytes();
    if (free_b < 0) { err = "cudaMemGetInfo"; return BL_E_CUDA; }
  }
  prof_.derive();
  std::vector<int64_t> avg;
  int64_t need = 0;
  for (int j = 0; j < nten(); ++j) {
    avg.push_back(prof_.ten[j].T / std::max<int64_t>(1, (int64_t)prof_.ten[j].k.size()));
    need += mem[j];
  }
  int r = 0;
  if (!colocatable(avg, span)) r = 1;
  else if (need > free_b) r = 2;
  *ok = r == 0;
  if (why) *why = r;
  return BL_OK;
}

bl_status Engine::reset(const bl_params* p, std::string& err) {
  bl_status st = stop(err);
  if (st != BL_OK && st != BL_E_CUDA) return st;
  if (p) {
    if (p->max_requests != prm_.max_requests) { err = "max_requests cannot change on reset"; return BL_E_INVALID; }
    if (p->barrier < 0 || p->barrier > 3) { err = "invalid bl_params.barrier"; return BL_E_INVALID; }
    prm_ = *p;
    prof_.g = prm_.sm_unit;
    prof_.derive();
  }
  const uint64_t n = next_id_.load();
  for (uint64_t i = 0; i < n && (int64_t)i < cap_; ++i) {
    reqs_[i].published.store(0);
    reqs_[i].done.store(0);
  }
  next_id_ = 0;
  n_done_ = 0;
  last_submit_arrival_.clear();
  failed_ = false;
  fail_msg_.clear();
  std::lock_guard<std::mutex> lk(log_mu_);
  dlog_.clear();
  llog_.clear();
  tlog_.clear();
  return BL_OK;
}

bl_status Engine::temporal_log(size_t first, bl_temporal_rec* buf, size_t cap, size_t* n) {
  std::lock_guard<std::mutex> lk(log_mu_);
  size_t c = 0;
  for (size_t i = first; i < tlog_.size() && c < cap; ++i) buf[c++] = tlog_[i];
  if (n) *n = (buf == nullptr) ? tlog_.size() : c;
  return BL_OK;
}

// Host cost of decide() (L436): the logged inputs of each record replayed reps
// times on this thread, timed with the steady clock.
bl_status Engine::time_decide(const bl_decision* recs, size_t n, int reps, int64_t* total_ns, int64_t* picks,
                              std::string& err) {
  if (!recs || reps < 1) { err = "bad args"; return BL_E_INVALID; }
  if (!prof_.complete()) { err = "profile incomplete"; return BL_E_STATE; }
  prof_.g = prm_.sm_unit;
  prof_.derive();
  std::vector<std::vector<ActiveReq>> in(n);
  for (size_t r = 0; r < n; ++r) {
    const bl_decision& d = recs[r];
    if (d.n_active < 1 || d.n_active > nten()) { err = "bad active set"; return BL_E_INVALID; }
    for (int i = 0; i < d.n_active; ++i) {
      const int t = d.act_tenant[i];
      if (t < 0 || t >= nten() || d.act_next[i] < 0 || d.act_next[i] >= (int)prof_.ten[t].k.size()) {
        err = "bad active entry";
        return BL_E_INVALID;
      }
      in[r].push_back({t, d.act_arrival[i], d.act_next[i]});
    }
  }
  SchedParams sp{prm_.squad_max, prm_.split_pct, prm_.seed_all != 0, prm_.ablate, prm_.squad_max_solo};
  Decision d;
  DecideScratch sc;
  int64_t np = 0;
  const int64_t t0 = now_ns();
  for (int rep = 0; rep < reps; ++rep)
    for (size_t r = 0; r < n; ++r) {
      decide(recs[r].now, in[r].data(), (int)in[r].size(), prof_, sp, d, sc);
      np += (int64_t)d.picks.size();
    }
  const int64_t t1 = now_ns();
  if (total_ns) *total_ns = t1 - t0;
  if (picks) *picks = np;
  return BL_OK;
}

bl_status Engine::decisions(size_t first, bl_decision* buf, size_t cap, size_t* n) {
  std::lock_guard<std::mutex> lk(log_mu_);
  size_t c = 0;
  for (size_t i = first; i < dlog_.size() && c < cap; ++i) buf[c++] = dlog_[i];
  if (n) *n = (buf == nullptr) ? dlog_.size() : c;
  return BL_OK;
}

bl_status Engine::launches(size_t first, bl_launch_rec* buf, size_t cap, size_t* n) {
  std::lock_guard<std::mutex> lk(log_mu_);
  size_t c = 0;
  for (size_t i = first; i < llog_.size() && c < cap; ++i) buf[c++] = llog_[i];
  if (n) *n = (buf == nullptr) ? llog_.size() : c;
  return BL_OK;
}

static void to_record(const Decision& d, bl_decision& r) {
  std::memset(&r, 0, sizeof(r));
  r.now = d.now;
  r.t_hat = d.t_hat;
  r.t_nsp = d.t_nsp;
  r.n_active = (int32_t)d.active.size();
  for (size_t i = 0; i < d.active.size() && i < BL_MAX_TENANTS; ++i) {
    r.act_tenant[i] = d.active[i].tenant;
    r.act_arrival[i] = d.active[i].arrival;
    r.act_next[i] = d.active[i].next;
  }
  r.n_part = (int32_t)d.parts.size();
  r.config_sp = d.sp ? 1 : 0;
  for (size_t i = 0; i < d.parts.size(); ++i) {
    r.part_tenant[i] = d.parts[i];
    r.part_p[i] = d.sp ? d.p[i] : 0;
  }
  r.n_picks = (int32_t)d.picks.size();
  for (size_t i = 0; i < d.picks.size() && i < BL_MAX_SQUAD; ++i) {
    r.pick_tenant[i] = d.picks[i].tenant;
    r.pick_kernel[i] = d.picks[i].kernel;
    r.pick_lo[i] = (int16_t)d.picks[i].lo;
    r.pick_hi[i] = (int16_t)d.picks[i].hi;
  }
}

bl_status Engine::decide_pure(int64_t now, int n, const int32_t* ten, const int64_t* arr, const int32_t* nxt,
                              bl_decision* out, std::string& err) {
  if (n < 1 || n > nten() || !ten || !arr || !nxt || !out) { err = "bad active set"; return BL_E_INVALID; }
  if (!prof_.complete()) { err = "profile incomplete"; return BL_E_STATE; }
  prof_.g = prm_.sm_unit;
  prof_.derive();
  std::vector<ActiveReq> a(n);
  std::vector<int> seen(nten(), 0);
  for (int i = 0; i < n; ++i) {
    if (ten[i] < 0 || ten[i] >= nten() || seen[ten[i]]++ || nxt[i] < 0 || nxt[i] >= (int)prof_.ten[ten[i]].k.size()) {
      err = "bad active entry";
      return BL_E_INVALID;
    }
    a[i] = {ten[i], arr[i], nxt[i]};
  }
  SchedParams sp{prm_.squad_max, prm_.split_pct, prm_.seed_all != 0, prm_.ablate, prm_.squad_max_solo};
  Decision d;
  DecideScratch sc;
  decide(now, a.data(), n, prof_, sp, d, sc);
  to_record(d, *out);
  return BL_OK;
}

// Participants (tenant-id order) and their kernels in pick order, validated.
static bool squad_of(const Profile& prof, int n, const int32_t* ten, const int32_t* ker, std::vector<int>& parts,
                     std::vector<std::vector<int>>& ks, std::string& err) {
  const int nt = (int)prof.ten.size();
  if (n < 1 || !ten || !ker) { err = "empty squad"; return false; }
  std::vector<std::vector<int>> by(nt);
  for (int i = 0; i < n; ++i) {
    if (ten[i] < 0 || ten[i] >= nt || ker[i] < 0 || ker[i] >= (int)prof.ten[ten[i]].k.size()) {
      err = "bad pick " + std::to_string(i);
      return false;
    }
    by[ten[i]].push_back(ker[i]);
  }
  parts.clear();
  ks.clear();
  for (int j = 0; j < nt; ++j)
    if (!by[j].empty()) { parts.push_back(j); ks.push_back(by[j]); }
  return true;
}

bl_status Engine::predict(int n, const int32_t* ten, const int32_t* ker, const int32_t* p, int64_t* out,
                          std::string& err) {
  if (!out) { err = "null out"; return BL_E_INVALID; }
  if (!prof_.complete()) { err = "profile incomplete"; return BL_E_STATE; }
  prof_.g = prm_.sm_unit;
  prof_.derive();
  std::vector<int> parts;
  std::vector<std::vector<int>> ks;
  if (!squad_of(prof_, n, ten, ker, parts, ks, err)) return BL_E_INVALID;
  if (!p) {
    *out = predict_nsp(prof_, parts, ks);
    return BL_OK;
  }
  std::vector<int> pv(p, p + parts.size());
  int sum = 0;
  for (int x : pv) {
    if (x < 1) { err = "every participant needs >= 1 partition"; return BL_E_INVALID; }
    sum += x;
  }
  if (sum != prof_.N) { err = "partitions must sum to N"; return BL_E_INVALID; }
  *out = predict_sp(prof_, parts, ks, pv);
  return BL_OK;
}

// One squad as given (f1 study): each participant's picks in order on its
// stream, every chain released by one event, every launch with the full exit
// protocol (start/end stamps); reps times, medians.
bl_status Engine::run_squad(int n, const int32_t* ten, const int32_t* ker, const int16_t* lo, const int16_t* hi,
                            int reps, int64_t* makespan, int64_t* kernel_ns, std::string& err) {
  if (!rt_) { err = "no device"; return BL_E_STATE; }
  if (started_) { err = "run_squad while running"; return BL_E_STATE; }
  if (n < 1 || !ten || !ker || !lo || !hi || reps < 1 || !makespan) { err = "bad args"; return BL_E_INVALID; }
  for (int i = 0; i < n; ++i)
    if (ten[i] < 0 || ten[i] >= nten() || ker[i] < 0 || ker[i] >= (int)ten_[ten[i]].handles.size() ||
        lo[i] < 0 || hi[i] > S() || lo[i] >= hi[i]) {
      err = "bad pick " + std::to_string(i);
      return BL_E_INVALID;
    }
  rt_->set_device();
  if (!temporal_stream_) temporal_stream_ = rt_->stream_create();
  void* go = rt_->event_create();
  std::vector<std::vector<int64_t>> kd(n);
  std::vector<int64_t> ms;
  std::vector<uint64_t> seqs(n);
  for (int r = 0; r < reps; ++r) {
    if (!rt_->device_sync()) { err = "device error"; rt_->event_destroy(go); return BL_E_CUDA; }
    rt_->event_record(go, temporal_stream_);
    std::vector<int> waited(nten(), 0);
    for (int i = 0; i < n; ++i) {
      TenantRT& t = ten_[ten[i]];
      if (!waited[ten[i]]) { rt_->stream_wait(t.stream, go); waited[ten[i]] = 1; }
      seqs[i] = rt_->launch(t.handles[ker[i]], lo[i], hi[i], t.stream, err, true);
      if (!seqs[i]) { rt_->event_destroy(go); return BL_E_CUDA; }
    }
    if (!rt_->device_sync()) { err = "device error"; rt_->event_destroy(go); return BL_E_CUDA; }
    rt_->refresh_sync(seqs.front(), seqs.back());
    int64_t a = INT64_MAX, b = 0;
    for (int i = 0; i < n; ++i) {
      LaunchStats st{};
      if (!rt_->poll(seqs[i], &st)) { err = "squad launch stats missing"; rt_->event_destroy(go); return BL_E_CUDA; }
      kd[i].push_back(st.end_host - st.start_host);
      a = std::min(a, st.start_host);
      b = std::max(b, st.end_host);
    }
    ms.push_back(b - a);
  }
  rt_->event_destroy(go);
  auto med = [](std::vector<int64_t> v) {
    std::sort(v.begin(), v.end());
    return v[v.size() / 2];
  };
  *makespan = med(ms);
  if (kernel_ns)
    for (int i = 0; i < n; ++i) kernel_ns[i] = med(kd[i]);
  return BL_OK;
}

void Engine::log_decision(const Decision& d) {
  bl_decision r;
  to_record(d, r);
  std::lock_guard<std::mutex> lk(log_mu_);
  dlog_.push_back(r);
}

// ------------------------------------------------------------------ scheduler thread
void Engine::scan_submissions() {
  const uint64_t hi = next_id_.load(std::memory_order_acquire);
  while (scan_ < hi && (int64_t)scan_ < cap_ && reqs_[scan_].published.load(std::memory_order_acquire)) {
    fifo_[reqs_[scan_].tenant].push_back(scan_);
    ++scan_;
  }
}

uint64_t Engine::launch_one(int t, int k, int lo, int hi, void* stream, int64_t req, bool last, bool stamp) {
  std::string err;
  TenantRT& tr = ten_[t];
  const bool own = stream == tr.stream;   // light-exit chaining only on the tenant's own stream
  if (!own) stamp = true;
  if (k == 0 && tr.in_bytes) {
    if (!rt_->memcpy_async(tr.dev_in, tr.host_in, tr.in_bytes, stream)) {
      fail("H2D input copy failed");
      return 0;
    }
    if (own) tr.prev_light = 0, tr.dep_seq = 0;
  }
  const uint64_t seq = rt_->alloc_seq();
  const int h = tr.handles[k];
  if (!rt_->launch_seq(h, seq, lo, hi, stream, err, stamp, own ? tr.prev_light : 0, own ? tr.dep_seq : 0,
                       tr.dep_tot)) {
    fail(err);
    return 0;
  }
  if (own) {
    tr.prev_light = stamp ? 0 : seq;
    tr.dep_seq = rt_->counts(h) ? seq : 0;
    tr.dep_tot = rt_->kernel(h).tiles;
  }
  bl_launch_rec rec{};
  rec.seq = seq;
  rec.tenant = t;
  rec.kernel = k;
  rec.lo = (int16_t)lo;
  rec.hi = (int16_t)hi;
  rec.req = req >= 0 ? (uint64_t)req : ~0ull;
  size_t idx;
  {
    std::lock_guard<std::mutex> lk(log_mu_);
    idx = llog_.size();
    llog_.push_back(rec);
  }
  if (last && tr.out_bytes) {
    // the request completes when its output has landed in host memory: a
    // one-CTA marker after the D2H copy carries the completion stamp
    if (!rt_->memcpy_async(tr.host_out, tr.dev_out, tr.out_bytes, stream)) {
      fail("D2H output copy failed");
      return 0;
    }
    const uint64_t mseq = rt_->launch_marker(stream, err);
    if (!mseq) {
      fail(err);
      return 0;
    }
    if (own) tr.prev_light = 0, tr.dep_seq = 0;
    pending_.push_back({seq, idx, req, k, 0});
    pending_.push_back({mseq, (size_t)-1, req, -1, 1});
    return seq;
  }
  if (stamp) pending_.push_back({seq, idx, req, k, last ? 1 : 0});
  return seq;
}

// ------------------------------------------------------------------ parallel launch
bool Engine::prepare_one(int t, int k, int lo, int hi, int64_t req, bool last, std::vector<LaunchItem>& items,
                         bool stamp) {
  const TenantRT& tr = ten_[t];
  if (k == 0 && tr.in_bytes) items.push_back({LaunchItem::H2D, 1, -1, 0, 0, 0});
  const uint64_t seq = rt_->alloc_seq();
  items.push_back({LaunchItem::KERNEL, (uint8_t)(stamp ? 1 : 0), tr.handles[k], seq, lo, hi});
  bl_launch_rec rec{};
  rec.seq = seq;
  rec.tenant = t;
  rec.kernel = k;
  rec.lo = (int16_t)lo;
  rec.hi = (int16_t)hi;
  rec.req = req >= 0 ? (uint64_t)req : ~0ull;
  size_t idx;
  {
    std::lock_guard<std::mutex> lk(log_mu_);
    idx = llog_.size();
    llog_.push_back(rec);
  }
  if (last && tr.out_bytes) {
    // the request completes when its output has landed in host memory: a
    // one-CTA marker after the D2H copy carries the completion stamp
    const uint64_t mseq = rt_->alloc_seq();
    items.push_back({LaunchItem::D2H, 1, -1, 0, 0, 0});
    items.push_back({LaunchItem::MARKER, 1, -1, mseq, 0, 0});
    pending_.push_back({seq, idx, req, k, 0});
    pending_.push_back({mseq, (size_t)-1, req, -1, 1});
  } else if (stamp) {
    pending_.push_back({seq, idx, req, k, last ? 1 : 0});
  }
  return true;
}

bool Engine::exec_items(int t, const std::vector<LaunchItem>& items, void* stream, std::string& err) {
  TenantRT& tr = ten_[t];
  for (const LaunchItem& it : items) {
    if (it.kind != LaunchItem::KERNEL) tr.prev_light = 0, tr.dep_seq = 0;
    switch (it.kind) {
      case LaunchItem::KERNEL:
        if (!rt_->launch_seq(it.handle, it.seq, it.lo, it.hi, stream, err, it.stamp != 0, tr.prev_light, tr.dep_seq,
                             tr.dep_tot))
          return false;
        tr.prev_light = it.stamp ? 0 : it.seq;
        tr.dep_seq = rt_->counts(it.handle) ? it.seq : 0;
        tr.dep_tot = rt_->kernel(it.handle).tiles;
        break;
      case LaunchItem::H2D:
        if (!rt_->memcpy_async(tr.dev_in, tr.host_in, tr.in_bytes, stream)) { err = "H2D input copy failed"; return false; }
        break;
      case LaunchItem::D2H:
        if (!rt_->memcpy_async(tr.host_out, tr.dev_out, tr.out_bytes, stream)) { err = "D2H output copy failed"; return false; }
        break;
      case LaunchItem::MARKER:
        if (!rt_->launch_marker_seq(it.seq, stream, err)) return false;
        break;
    }
  }
  return true;
}

void Engine::push_job(int t, LaunchJob&& job) {
  Launcher& L = *launchers_[t];
  {
    std::lock_guard<std::mutex> lk(L.mu);
    L.q.push_back(std::move(job));
  }
  L.queued.fetch_add(1, std::memory_order_release);
}

void Engine::launcher_main(int t) {
  rt_->set_device();
  Launcher& L = *launchers_[t];
  std::string err;
  for (;;) {
    if (L.queued.load(std::memory_order_acquire) == 0) {
      if (L.quit.load()) return;
      cpu_relax();
      continue;
    }
    LaunchJob job;
    {
      std::lock_guard<std::mutex> lk(L.mu);
      job = std::move(L.q.front());
      L.q.pop_front();
    }
    L.queued.fetch_sub(1, std::memory_order_release);
    if (job.wait_squad) {
      // squad barrier: the previous squad's events must have been recorded
      // (by their launchers) before this stream waits on them
      for (size_t i = 0; i < job.wait_parts.size(); ++i) {
        const int l = job.wait_parts[i];
        const uint64_t need = job.wait_sq.empty() ? job.wait_squad : job.wait_sq[i];
        while (launchers_[l]->recorded.load(std::memory_order_acquire) < need) {
          if (L.quit.load() || failed_) return;
          cpu_relax();
        }
      }
      // the previous squad's event on this tenant's own stream is already
      // ordered by the stream: waiting on it would only cut the programmatic
      // (PDL) overlap between this stream's consecutive kernels
      for (size_t i = 0; i < job.wait_events.size(); ++i)
        if (i >= job.wait_parts.size() || job.wait_parts[i] != t) rt_->stream_wait(ten_[t].stream, job.wait_events[i]);
    }
    if (!exec_items(t, job.items, ten_[t].stream, err)) {
      fail(err);
      return;
    }
    if (job.record_event) rt_->event_record(job.record_event, ten_[t].stream);
    if (job.squad) L.recorded.store(job.squad, std::memory_order_release);
  }
}

void Engine::start_launchers() {
  launchers_.clear();
  if (!use_launchers() || !par_launch_) return;
  for (int j = 0; j < nten(); ++j) launchers_.emplace_back(new Launcher());
  for (int j = 0; j < nten(); ++j) launchers_[j]->th = std::thread([this, j] { launcher_main(j); });
}

void Engine::stop_launchers() {
  for (auto& L : launchers_) L->quit = true;
  for (auto& L : launchers_)
    if (L->th.joinable()) L->th.join();
  launchers_.clear();
}

void Engine::harvest() {
  if (!rt_ || pending_.empty()) return;
  if (!harvest_all_) {
    // mirror the pending launches' stats (copy engine), at most every 25 us
    const int64_t t = now_ns();
    if (t - last_refresh_ns_ >= 25000) {
      rt_->refresh_async(pending_.front().seq, pending_.back().seq);
      last_refresh_ns_ = t;
    }
  }
  size_t w = 0;
  for (size_t i = 0; i < pending_.size(); ++i) {
    PendingLaunch& p = pending_[i];
    LaunchStats st;
    if (!rt_->poll(p.seq, &st)) {
      pending_[w++] = p;
      continue;
    }
    if (p.log_idx != (size_t)-1) {
      std::lock_guard<std::mutex> lk(log_mu_);
      bl_launch_rec& r = llog_[p.log_idx];
      r.start_ns = st.start_host;
      r.end_ns = st.end_host;
      r.nsm = st.nsm;
      r.fallback = st.fallback;
      for (int i = 0; i < 8; ++i) r.sm_mask[i] = st.mask[i];
    }
    if (p.req >= 0) {
      Req& q = reqs_[p.req];
      if (p.kernel == 0) q.start = st.start_host;
      if (p.last) {
        q.finish = st.end_host;
        q.done.store(1, std::memory_order_release);
        n_done_.fetch_add(1);
      }
    }
  }
  pending_.resize(w);
}

void Engine::retire_inflight() {
  while (!inflight_.empty()) {
    // an event not yet recorded (its launcher is behind) queries as complete
    if (!launchers_.empty())
      for (int l : inflight_.front().parts)
        if (launchers_[l]->recorded.load(std::memory_order_acquire) < inflight_.front().squad) return;
    bool all = true;
    for (void* e : inflight_.front().events) {
      const int q = rt_->event_query(e);
      if (q < 0) {
        fail("device error (event query)");
        return;
      }
      if (q == 0) { all = false; break; }
    }
    if (!all) return;
    inflight_.pop_front();
  }
}

void Engine::thread_main() {
  if (rt_) rt_->set_device();
  switch (prm_.policy) {
    case BL_POLICY_BLESS: loop_bless(); break;
    case BL_POLICY_ISO:
    case BL_POLICY_STATIC: loop_at_arrival(false); break;
    case BL_POLICY_UNBOUND: loop_at_arrival(true); break;
    case BL_POLICY_TEMPORAL: loop_temporal(); break;
    default: fail("unknown policy");
  }
  // keep harvesting completions until stopped
  while (!stop_) {
    if (rt_) harvest();
    std::this_thread::sleep_for(std::chrono::microseconds(20));
  }
}

// BLESS: squads on the event-barriered tenant streams (§4.3-§4.5).
int Engine::solo_inflight_tenant() const {
  if (inflight_.empty()) return -1;
  const int l = inflight_.front().parts.empty() ? -1 : inflight_.front().parts[0];
  for (const Inflight& f : inflight_)
    if (!f.solo_nsp || f.parts.size() != 1 || f.parts[0] != l) return -1;
  return l;
}

void Engine::launch_squad(const Decision& d, const std::vector<int64_t>& act_req, const std::vector<int>& act_next,
                          bool join_solo) {
  (void)act_next;
  // Squad barrier: every participant waits for the previous squad's kernels
  // (the paper synchronises after each squad, L276; here a GPU-side event
  // wait instead of a host synchronisation, L432's 20 us switch).
  const uint64_t sq = ++squad_id_;
  // full exit protocol only where the host observes completion: a request's
  // first/last kernel and the last kernel of each participant's chain
  std::vector<int> last_pick(nten(), -1);
  for (size_t i = 0; i < d.picks.size(); ++i) last_pick[d.picks[i].tenant] = (int)i;
  auto stamp_of = [&](size_t i) {
    const Pick& p = d.picks[i];
    return p.kernel == 0 || p.kernel == (int)prof_.ten[p.tenant].k.size() - 1 || last_pick[p.tenant] == (int)i;
  };
  // What each participant's chain waits for.  barrier = 0 (paper-literal,
  // L276): every other participant of the previous squad.  barrier = 1
  // (reading R37): the latest chain of every other tenant that is still in
  // flight and whose kernels ran on logical SMs this participant's kernels
  // will use -- per SM the squads still run one after the other, but a chain
  // no longer waits for chains on SMs it does not touch.
  const int nt = nten();
  const bool rbar = (prm_.barrier & 1) != 0;
  // (the paper-literal barrier keeps the scheduler thread's per-squad work
  // minimal: no masks, no per-participant lists)
  std::vector<std::array<uint64_t, 3>> umask(rbar ? nt : 0, std::array<uint64_t, 3>{0, 0, 0});
  std::vector<std::vector<int>> wparts(rbar ? nt : 0);
  std::vector<std::vector<void*>> wevs(rbar ? nt : 0);
  std::vector<std::vector<uint64_t>> wsqs(rbar ? nt : 0);
  if (rbar) {
    auto setbits = [](std::array<uint64_t, 3>& m, int lo, int hi) {
      for (int w = 0; w < 3; ++w) {
        const int a = std::max(lo, 64 * w), b = std::min(hi, 64 * w + 64);
        if (a < b) m[w] |= (b - a == 64 ? ~0ull : ((1ull << (b - a)) - 1)) << (a - 64 * w);
      }
    };
    for (const Pick& p : d.picks) setbits(umask[p.tenant], p.lo, p.hi);
    if ((int)last_chain_.size() != nt) last_chain_.assign(nt, LastChain{});
  }
  if (rbar)
    for (int j : d.parts)
      for (int l = 0; l < nt; ++l) {
        const LastChain& c = last_chain_[l];
        if (l == j || !c.ev) continue;
        if (inflight_.empty() || c.squad < inflight_.front().squad) continue;   // retired: complete
        if (!((c.mask[0] & umask[j][0]) | (c.mask[1] & umask[j][1]) | (c.mask[2] & umask[j][2]))) continue;
        wparts[j].push_back(l);
        wevs[j].push_back(c.ev);
        wsqs[j].push_back(c.squad);
      }
  if (join_solo) {   // R38: the arrival does not wait for the in-flight solo squads
    wparts.assign(nt, {});
    wevs.assign(nt, {});
    wsqs.assign(nt, {});
  }
  if (launchers_.empty()) {   // single launch thread (BLESS_LAUNCH_THREADS=0)
    for (int j : d.parts) {
      if (rbar || join_solo) {   // (join_solo: the lists were cleared above)
        for (void* e : wevs[j]) rt_->stream_wait(ten_[j].stream, e);
      } else {
        for (size_t i = 0; i < prev_events_.size(); ++i)   // own stream: already ordered (see launcher_main)
          if (i >= prev_parts_.size() || prev_parts_[i] != j) rt_->stream_wait(ten_[j].stream, prev_events_[i]);
      }
      ten_[j].prev_light = 0;
    }
    for (size_t i = 0; i < d.picks.size(); ++i) {
      const Pick& p = d.picks[i];
      const int j = p.tenant, k = p.kernel;
      const bool last = k == (int)prof_.ten[j].k.size() - 1;
      if (!launch_one(j, k, p.lo, p.hi, ten_[j].stream, (k == 0 || last) ? act_req[j] : -1, last, stamp_of(i))) return;
    }
  }
  std::vector<LaunchJob> jobs(launchers_.empty() ? 0 : nten());
  if (!launchers_.empty()) {
    for (int j : d.parts) {
      jobs[j].squad = sq;
      if (rbar || join_solo) {
        jobs[j].wait_squad = wparts[j].empty() ? 0 : 1;
        jobs[j].wait_parts = std::move(wparts[j]);
        jobs[j].wait_sq = std::move(wsqs[j]);
        jobs[j].wait_events = std::move(wevs[j]);
      } else {
        jobs[j].wait_squad = prev_squad_;
        jobs[j].wait_parts = prev_parts_;
        jobs[j].wait_events = prev_events_;
      }
    }
    for (size_t i = 0; i < d.picks.size(); ++i) {
      const Pick& p = d.picks[i];
      const int j = p.tenant, k = p.kernel;
      const bool last = k == (int)prof_.ten[j].k.size() - 1;
      prepare_one(j, k, p.lo, p.hi, (k == 0 || last) ? act_req[j] : -1, last, jobs[j].items, stamp_of(i));
    }
  }
  Inflight inf;
  inf.squad = sq;
  inf.parts = d.parts;
  inf.solo_nsp = d.parts.size() == 1 && !d.sp;
  for (int j : d.parts) {
    TenantRT& t = ten_[j];
    void* ev = t.events[t.ev_next++ % t.events.size()];
    if (launchers_.empty()) rt_->event_record(ev, t.stream);
    else jobs[j].record_event = ev;
    inf.events.push_back(ev);
  }
  for (int j : d.parts)
    if (!launchers_.empty()) push_job(j, std::move(jobs[j]));
  for (size_t i = 0; rbar && i < d.parts.size(); ++i) {
    LastChain& c = last_chain_[d.parts[i]];
    c.ev = inf.events[i];
    c.squad = sq;
    for (int w = 0; w < 3; ++w) c.mask[w] = umask[d.parts[i]][w];
  }
  prev_events_ = inf.events;
  prev_parts_ = d.parts;
  prev_squad_ = sq;
  inflight_.push_back(std::move(inf));
}

void Engine::loop_bless() {
  const bool virt = prm_.clock == BL_CLOCK_VIRTUAL;
  const int nt = nten();
  std::vector<int64_t> act_req(nt, -1);
  std::vector<int> act_next(nt, 0);
  std::vector<ActiveReq> av;
  SchedParams sp{prm_.squad_max, prm_.split_pct, prm_.seed_all != 0, prm_.ablate, prm_.squad_max_solo};
  int64_t vnow = 0;   // VIRTUAL clock
  int64_t E = 0;      // WALL: predicted end of the last launched squad
  bool join_solo = false;   // WALL, R38: this decision joins in-flight solo squads
  const size_t max_inflight = (size_t)std::max(1, prm_.max_inflight_squads);
  while (!stop_) {
    if (rt_) {
      harvest();
      retire_inflight();
      if (failed_) return;
    }
    scan_submissions();
    int64_t now;
    if (virt) {
      for (int j = 0; j < nt; ++j)
        if (act_req[j] < 0 && !fifo_[j].empty() && reqs_[fifo_[j].front()].arrival <= vnow) {
          act_req[j] = (int64_t)fifo_[j].front();
          act_next[j] = 0;
          fifo_[j].pop_front();
        }
      bool any = false;
      for (int j = 0; j < nt; ++j) any |= act_req[j] >= 0;
      if (!any) {
        int64_t nxt = INT64_MAX;
        for (int j = 0; j < nt; ++j)
          if (!fifo_[j].empty()) nxt = std::min(nxt, reqs_[fifo_[j].front()].arrival);
        if (nxt == INT64_MAX) return;  // trace finished (all submitted before start)
        vnow = nxt;
        continue;
      }
      now = vnow;
    } else {
      const int64_t host = now_ns();
      const bool gpu_idle = inflight_.empty();
      join_solo = false;
      if (!gpu_idle && (inflight_.size() >= max_inflight || host < E - prm_.lookahead_ns)) {
        // R38 (barrier bit 1; L57 "shrinks its resources instantly when other
        // requests arrive"): a request arriving while the GPU runs nothing but
        // another tenant's solo NSP squads is decided now and its chain starts
        // at once, beside the solo kernels (no preemption: they keep running,
        // sharing the SMs through their tile queues)
        const int l = (prm_.barrier & 2) ? solo_inflight_tenant() : -1;
        bool arrival = false;
        if (l >= 0 && inflight_.size() <= max_inflight)
          for (int j = 0; j < nt && !arrival; ++j)
            arrival = j != l && act_req[j] < 0 && !fifo_[j].empty() && reqs_[fifo_[j].front()].arrival <= host;
        if (!arrival) {
          cpu_relax();
          continue;
        }
        join_solo = true;
      }
      for (int j = 0; j < nt; ++j)
        if (act_req[j] < 0 && !fifo_[j].empty() && reqs_[fifo_[j].front()].arrival <= host) {
          act_req[j] = (int64_t)fifo_[j].front();
          act_next[j] = 0;
          fifo_[j].pop_front();
        }
      bool any = false;
      for (int j = 0; j < nt; ++j) any |= act_req[j] >= 0;
      if (!any) {
        cpu_relax();
        continue;
      }
      now = (gpu_idle || join_solo) ? host : std::max(host, E);
    }
    av.clear();
    for (int j = 0; j < nt; ++j)
      if (act_req[j] >= 0) av.push_back({j, reqs_[act_req[j]].arrival, act_next[j]});
    decide(now, av.data(), (int)av.size(), prof_, sp, dec_, scratch_);
    log_decision(dec_);
    if (rt_) {
      if (virt) {
        // a squad is not launched before the wall time of its newest arrival (R17)
        int64_t newest = INT64_MIN;
        for (int j : dec_.parts) newest = std::max(newest, reqs_[act_req[j]].arrival);
        for (int j : dec_.parts) reqs_[act_req[j]].arrival_host = t0_ + reqs_[act_req[j]].arrival;
        while (!stop_ && (now_ns() < t0_ + newest || inflight_.size() >= max_inflight)) {
          harvest();
          retire_inflight();
          if (failed_) return;
          cpu_relax();
        }
      }
      launch_squad(dec_, act_req, act_next, join_solo);
      if (failed_) return;
    }
    // advance the requests
    for (size_t i = 0; i < dec_.parts.size(); ++i) {
      const int j = dec_.parts[i];
      int c = 0;
      for (const Pick& p : dec_.picks) c += p.tenant == j;
      Req& r = reqs_[act_req[j]];
      if (!rt_ && act_next[j] == 0) r.start = now;
      act_next[j] += c;
      if (act_next[j] == (int)prof_.ten[j].k.size()) {
        if (!rt_) {  // model completion (device-less ctx): SURVEY C-3
          r.finish = now + dec_.chain_end[i];
          r.done.store(1, std::memory_order_release);
          n_done_.fetch_add(1);
        }
        act_req[j] = -1;
        act_next[j] = 0;
      }
    }
    if (virt) vnow = now + dec_.t_hat + prm_.squad_overhead_ns;
    else E = join_solo ? std::max(E, now + dec_.t_hat) : now + dec_.t_hat;
  }
}

// ISO / STATIC / UNBOUND: the whole request is launched at arrival on the
// tenant's stream, confined to its quota range or unrestricted (L103, L300).
void Engine::loop_at_arrival(bool unbound) {
  const int nt = nten();
  while (!stop_) {
    harvest();
    if (failed_) return;
    scan_submissions();
    const int64_t host = now_ns();
    bool launched = false;
    for (int j = 0; j < nt; ++j) {
      while (!fifo_[j].empty() && reqs_[fifo_[j].front()].arrival <= host) {
        const int64_t r = (int64_t)fifo_[j].front();
        fifo_[j].pop_front();
        const int m = (int)prof_.ten[j].k.size();
        const int lo = unbound ? 0 : ten_[j].lo, hi = unbound ? S() : ten_[j].hi;
        if (!launchers_.empty()) {
          LaunchJob job;
          for (int k = 0; k < m; ++k)
            prepare_one(j, k, lo, hi, (k == 0 || k == m - 1) ? r : -1, k == m - 1, job.items, k == 0 || k == m - 1);
          push_job(j, std::move(job));
        } else {
          for (int k = 0; k < m; ++k)
            if (!launch_one(j, k, lo, hi, ten_[j].stream, (k == 0 || k == m - 1) ? r : -1, k == m - 1,
                            k == 0 || k == m - 1))
              return;
        }
        launched = true;
      }
    }
    if (!launched) cpu_relax();
  }
}

// TEMPORAL (R22): slices of quota*P on the full GPU, one kernel at a time on a
// shared stream; non-preemptive, a kernel starts only if it is predicted to end
// inside the slice (except the slice's first kernel).  T-cap: fixed cyclic
// slices (idle slices stay idle).  T-wc: round robin skipping idle tenants.
void Engine::loop_temporal() {
  const int nt = nten();
  const int64_t P = std::max<int64_t>(1000, prm_.temporal_period_ns);
  std::vector<int64_t> len(nt), off(nt);
  int64_t acc = 0;
  for (int j = 0; j < nt; ++j) {
    len[j] = P * ten_[j].ppm / 1000000;
    off[j] = acc;
    acc += len[j];
  }
  std::vector<int64_t> act_req(nt, -1);
  std::vector<int> act_next(nt, 0);
  const int64_t base = now_ns();
  int64_t F = 0;                 // predicted time the GPU becomes free
  int64_t last_sid = -1;
  // T-wc turn state
  int turn = -1;
  int64_t turn_end = 0, sid_wc = 0;
  auto activate = [&](int j, int64_t host) {
    if (act_req[j] < 0 && !fifo_[j].empty() && reqs_[fifo_[j].front()].arrival <= host) {
      act_req[j] = (int64_t)fifo_[j].front();
      act_next[j] = 0;
      fifo_[j].pop_front();
    }
    return act_req[j] >= 0;
  };
  while (!stop_) {
    harvest();
    if (failed_) return;
    scan_submissions();
    const int64_t host = now_ns();
    int j = -1;
    int64_t slice_end = 0, sid = 0;
    // decision inputs for the log (bl_temporal_rec): which tenants have work
    // now, and the T-wc turn state before this iteration
    int32_t work_mask = 0;
    for (int q = 0; q < nt; ++q)
      if (act_req[q] >= 0 || (!fifo_[q].empty() && reqs_[fifo_[q].front()].arrival <= host)) work_mask |= 1 << q;
    const int rec_turn = turn;
    const int64_t rec_turn_end = turn_end;
    if (!prm_.temporal_work_conserving) {
      const int64_t cyc = (host - base) / P, pos = (host - base) % P;
      for (int q = 0; q < nt; ++q)
        if (pos >= off[q] && pos < off[q] + len[q]) j = q;
      if (j < 0) { cpu_relax(); continue; }
      slice_end = base + cyc * P + off[j] + len[j];
      sid = cyc * nt + j;
      if (!activate(j, host)) { cpu_relax(); continue; }
    } else {
      if (turn < 0 || host >= turn_end || !activate(turn, host)) {
        int pick = -1;
        for (int s = 1; s <= nt; ++s) {
          const int q = ((turn < 0 ? -1 : turn) + s + nt) % nt;
          if (activate(q, host)) { pick = q; break; }
        }
        if (pick < 0) { turn = -1; cpu_relax(); continue; }
        turn = pick;
        // the turn starts when the GPU is free (the oracle DES, des.run_temporal)
        turn_end = std::max(host, F) + len[pick];
        ++sid_wc;
      }
      j = turn;
      slice_end = turn_end;
      sid = sid_wc;
    }
    const int k = act_next[j];
    const int m = (int)prof_.ten[j].k.size();
    const int64_t dur = prof_.t(j, k, S());
    const int64_t st = std::max(F, host);
    const bool first = sid != last_sid;
    if (st < slice_end && (first || st + dur <= slice_end)) {
      bl_temporal_rec rec{};
      rec.t = host - base;
      rec.gpu_free = F - base;
      rec.slice_end = slice_end - base;
      rec.dur = dur;
      rec.sid = sid;
      rec.last_sid = last_sid;
      rec.turn = prm_.temporal_work_conserving ? rec_turn : -1;
      rec.turn_end = prm_.temporal_work_conserving && rec_turn >= 0 ? rec_turn_end - base : 0;
      rec.work_mask = work_mask;
      rec.tenant = j;
      rec.kernel = k;
      rec.work_conserving = prm_.temporal_work_conserving ? 1 : 0;
      {
        std::lock_guard<std::mutex> lk(log_mu_);
        tlog_.push_back(rec);
      }
      if (!launch_one(j, k, 0, S(), temporal_stream_, (k == 0 || k == m - 1) ? act_req[j] : -1, k == m - 1)) return;
      F = st + dur;
      last_sid = sid;
      if (++act_next[j] == m) {
        act_req[j] = -1;
        act_next[j] = 0;
      }
    } else {
      // T-wc: a kernel that does not fit ends the turn at once (the next
      // tenant with work takes over; des.run_temporal); T-cap idles to the
      // end of the fixed slice
      if (prm_.temporal_work_conserving) turn_end = host;
      cpu_relax();
    }
  }
}

}  // namespace bless
