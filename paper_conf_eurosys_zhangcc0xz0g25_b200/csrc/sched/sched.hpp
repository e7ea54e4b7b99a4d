// sched.hpp -- BLESS runtime scheduling decision, pure C++17 (no CUDA).
//
// PAPER.md §4.3 (multi-task scheduler, L173-L189) and §4.4 (execution
// configuration determiner, L191-L237), §4.5.2 (Semi-SP split, L253-L255).
// Readings R1-R18 are listed in DESIGN.md §3.  All decision arithmetic is
// integer (int64 / __int128) so the result is bit-exact and independent of
// libm; the argmin over spatial splits is an exact dynamic programme over
// suffixes instead of the oracle's plain enumeration.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

namespace bless {

// Quota -> SMs by largest remainder (R18).  ppm: quotas in parts per million.
std::vector<int> hamilton(const std::vector<int64_t>& ppm, int S);

struct KernelProfile {
  std::string name;
  int d = 0;                  // distinct SMs used unrestricted (L157 "d%", R19)
  std::vector<int64_t> t;     // t[s-1]: duration on s SMs, s = 1..S (L157, R11)
};

struct TenantProfile {
  std::string name;
  int64_t quota_ppm = 0;
  std::vector<KernelProfile> k;
  // derived
  int quota_sms = 0;
  std::vector<int64_t> tau;   // tau[k] = sum_{i<=k} t[i][quota_sms] (L157)
  int64_t T = 0;              // isolated latency T[n%] (L157)
  // SLO mode (§6.5: "replacing the isolated latency T[n%] in §4.3.1
  // with the required QoS target"): slo_ns > 0 replaces T in P_r = t_e/T, so
  // P~ = t_e / (tau * slo / T); the progress order compares t_e against
  // tau_prog[k] = floor(tau[k] * slo_ns / T) (reading R30).  slo_ns = 0:
  // tau_prog = tau (the paper's default, pace = isolated latency).
  int64_t slo_ns = 0;
  std::vector<int64_t> tau_prog;
  // Memory-management kernels (L229: "the durations of memory management
  // kernels (e.g., H2D, D2H memcpy) are added" in both predictors): the
  // request's input copy before kernel 0 and output copy after its last
  // kernel, profiled on the copy engine (ns, independent of the SM count).
  // Reading R31: Eq. 1 adds io_in / io_out to a participant's chain when its
  // picks include kernel 0 / the last kernel; Eq. 2 adds them to the level of
  // that kernel.  0 = no per-request host I/O.
  int64_t io_in = 0, io_out = 0;
  // Measured progress (reading R35): tau[n%][k] is "the
  // duration from the beginning of the application to the end of k" and
  // T[n%] its "isolated latency" -- measured along an isolated run of the
  // whole request on tau_sms SMs.  When tau_sms equals the tenant's quota
  // SMs, derive() takes tau (and T = tau.back()) from here instead of the
  // prefix sums of the per-kernel t[k][quota_sms].  Empty = not measured.
  int tau_sms = 0;
  std::vector<int64_t> tau_meas;
};

struct Profile {
  int S = 0, g = 4, N = 0;
  std::vector<TenantProfile> ten;
  void derive();              // quota_sms, tau, T, N
  int64_t t(int j, int k, int s) const { return ten[j].k[k].t[s - 1]; }
  bool complete() const;      // every kernel has S entries
};

bool load_profile_text(const std::string& path, Profile& out, std::string& err);
bool save_profile_text(const std::string& path, const Profile& p, std::string& err);

struct SchedParams {
  int squad_max = 50;   // R5
  int split_pct = 50;   // R16
  bool seed_all = true; // R6
  int ablate = 0;       // §6.8 ablation (R32): bit0 no multi-task scheduler, bit1 no determiner
  int squad_max_solo = 0;  // R36: cap of a squad with ONE active request (0 = squad_max)
};

struct ActiveReq {
  int tenant;
  int64_t arrival;
  int next;             // next kernel index of the request
};

struct Pick {
  int tenant, kernel, lo, hi;
};

struct Decision {
  int64_t now = 0, t_hat = 0, t_nsp = 0;
  std::vector<ActiveReq> active;      // sorted by tenant
  std::vector<Pick> picks;            // in pick order
  std::vector<int> parts;             // participants, sorted tenant ids
  bool sp = false;
  std::vector<int> p;                 // partitions per participant (SP)
  std::vector<int64_t> chain_end;     // per participant: predicted end of its picks
};

// Workspace reused across calls (no allocation on the hot path after warm-up).
struct DecideScratch {
  std::vector<int> nxt, order;
  std::vector<int64_t> arr;
  std::vector<std::vector<int>> ks;   // per participant kernel list
  std::vector<int64_t> Sj;            // K x (N+1) chain sums
  std::vector<int64_t> F;             // K x (N+1) DP table
};

void decide(int64_t now, const ActiveReq* act, int n_act, const Profile& prof, const SchedParams& prm,
            Decision& out, DecideScratch& scratch);

// The two squad-duration predictors for a GIVEN squad and configuration (the
// f1 predictor study, PAPER.md L214/L227/L237): parts = participants in
// tenant-id order, ks[i] = participant i's kernels in pick order.
int64_t predict_nsp(const Profile& prof, const std::vector<int>& parts, const std::vector<std::vector<int>>& ks);
int64_t predict_sp(const Profile& prof, const std::vector<int>& parts, const std::vector<std::vector<int>>& ks,
                   const std::vector<int>& p);

// Deployment (§4.2.2; reading R33): co-location rule and
// the central controller's tenant -> GPU placement.  avg[j] = average kernel
// duration (ns); span_x = largest / smallest allowed (L163: 10-300 us -> 30).
bool colocatable(const std::vector<int64_t>& avg, int64_t span_x);
std::vector<int> place(const std::vector<int64_t>& mem, const std::vector<int64_t>& avg,
                       const std::vector<int64_t>& gpu_free, int64_t span_x);

}  // namespace bless
