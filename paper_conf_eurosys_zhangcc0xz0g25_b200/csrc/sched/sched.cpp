// sched.cpp -- see sched.hpp.  Paper citations are PAPER.md lines.
#include "sched.hpp"

#include <algorithm>
#include <climits>
#include <fstream>
#include <sstream>

namespace bless {

static constexpr int64_t kPPM = 1000000;

std::vector<int> hamilton(const std::vector<int64_t>& ppm, int S) {
  // R18: seats H = round-half-up(S * sum / 1e6) (<= S); floors first, then the
  // leftover seats to the largest remainders, ties to the smaller tenant id.
  int64_t total = 0;
  for (int64_t q : ppm) total += q;
  int64_t H = std::min<int64_t>(S, (S * total + kPPM / 2) / kPPM);
  const int n = (int)ppm.size();
  std::vector<int> seats(n);
  std::vector<int64_t> rem(n);
  int64_t used = 0;
  for (int j = 0; j < n; ++j) {
    int64_t e = (int64_t)S * ppm[j];
    seats[j] = (int)(e / kPPM);
    rem[j] = e % kPPM;
    used += seats[j];
  }
  std::vector<int> idx(n);
  for (int j = 0; j < n; ++j) idx[j] = j;
  std::stable_sort(idx.begin(), idx.end(), [&](int a, int b) { return rem[a] > rem[b]; });
  for (int64_t i = 0; i < H - used && i < n; ++i) seats[idx[i]] += 1;
  return seats;
}

void Profile::derive() {
  N = g > 0 ? S / g : 0;
  std::vector<int64_t> ppm;
  for (auto& tn : ten) ppm.push_back(tn.quota_ppm);
  std::vector<int> qs = hamilton(ppm, S);
  for (size_t j = 0; j < ten.size(); ++j) {
    auto& tn = ten[j];
    tn.quota_sms = qs[j];
    tn.tau.assign(tn.k.size(), 0);
    int64_t acc = 0;
    for (size_t k = 0; k < tn.k.size(); ++k) {
      if ((int)tn.k[k].t.size() == S && tn.quota_sms >= 1) acc += tn.k[k].t[tn.quota_sms - 1];
      tn.tau[k] = acc;
    }
    if (!tn.tau_meas.empty() && tn.tau_meas.size() == tn.k.size() && tn.tau_sms == tn.quota_sms) {
      tn.tau = tn.tau_meas;   // R35: measured along an isolated run at the quota
      acc = tn.tau.back();
    }
    tn.T = acc;
    tn.tau_prog = tn.tau;
    if (tn.slo_ns > 0 && tn.T > 0)
      for (size_t k = 0; k < tn.k.size(); ++k)
        tn.tau_prog[k] = (int64_t)(((__int128)tn.tau[k] * tn.slo_ns) / tn.T);
  }
}

bool Profile::complete() const {
  for (auto& tn : ten)
    for (auto& k : tn.k)
      if ((int)k.t.size() != S || k.d < 1) return false;
  return S > 0;
}

bool load_profile_text(const std::string& path, Profile& out, std::string& err) {
  std::ifstream f(path);
  if (!f) { err = "cannot open " + path; return false; }
  std::string a, b;
  int ver = 0;
  f >> a >> ver;
  if (a != "bless-profile" || ver != 1) { err = "bad profile header"; return false; }
  Profile p;
  int n = 0;
  f >> a >> p.S >> b >> p.g;
  if (a != "S" || b != "g" || p.S <= 0 || p.g <= 0) { err = "bad S/g line"; return false; }
  f >> a >> n;
  if (a != "tenants" || n < 0) { err = "bad tenants line"; return false; }
  for (int j = 0; j < n; ++j) {
    TenantProfile tn;
    int m = 0;
    f >> a >> tn.name >> tn.quota_ppm >> m;
    if (a != "tenant" || m < 0) { err = "bad tenant line"; return false; }
    for (;;) {  // optional "slo <ns>" (SLO mode, R30) and "io <in_ns> <out_ns>" (R31) lines
      const std::streampos pos = f.tellg();
      if (!(f >> a)) { f.clear(); f.seekg(pos); break; }
      if (a == "slo") {
        f >> tn.slo_ns;
        if (!f || tn.slo_ns < 0) { err = "bad slo line"; return false; }
      } else if (a == "io") {
        f >> tn.io_in >> tn.io_out;
        if (!f || tn.io_in < 0 || tn.io_out < 0) { err = "bad io line"; return false; }
      } else if (a == "tau") {   // measured progress (R35): tau <sms> <tau_0> .. <tau_{m-1}>
        f >> tn.tau_sms;
        tn.tau_meas.resize(m);
        for (int k = 0; k < m; ++k) f >> tn.tau_meas[k];
        if (!f || tn.tau_sms < 1) { err = "bad tau line"; return false; }
        for (int k = 0; k < m; ++k)
          if (tn.tau_meas[k] < 0 || (k && tn.tau_meas[k] < tn.tau_meas[k - 1])) { err = "tau not monotone"; return false; }
      } else {
        f.seekg(pos);
        break;
      }
    }
    for (int k = 0; k < m; ++k) {
      KernelProfile kp;
      f >> a >> kp.name >> kp.d;
      if (a != "kernel") { err = "bad kernel line"; return false; }
      kp.t.resize(p.S);
      for (int s = 0; s < p.S; ++s) f >> kp.t[s];
      if (!f) { err = "truncated kernel line"; return false; }
      tn.k.push_back(std::move(kp));
    }
    p.ten.push_back(std::move(tn));
  }
  p.derive();
  out = std::move(p);
  return true;
}

bool save_profile_text(const std::string& path, const Profile& p, std::string& err) {
  std::ofstream f(path);
  if (!f) { err = "cannot write " + path; return false; }
  f << "bless-profile 1\nS " << p.S << " g " << p.g << "\ntenants " << p.ten.size() << "\n";
  for (auto& tn : p.ten) {
    f << "tenant " << tn.name << " " << tn.quota_ppm << " " << tn.k.size() << "\n";
    if (tn.slo_ns > 0) f << "slo " << tn.slo_ns << "\n";
    if (tn.io_in > 0 || tn.io_out > 0) f << "io " << tn.io_in << " " << tn.io_out << "\n";
    if (!tn.tau_meas.empty()) {
      f << "tau " << tn.tau_sms;
      for (int64_t v : tn.tau_meas) f << " " << v;
      f << "\n";
    }
    for (auto& k : tn.k) {
      f << "kernel " << k.name << " " << k.d;
      for (int64_t v : k.t) f << " " << v;
      f << "\n";
    }
  }
  return (bool)f;
}

// ---------------------------------------------------------------------------
// §4.3.1 progress order (L177-L179).  x is "more behind" than y iff, in order:
//   ratio t_e/tau larger (tau == 0 counts as +inf, R3), compared exactly by
//   cross multiplication in 128 bits (R1, R2); then smaller tau; earlier
//   arrival; smaller tenant id (R4).  This is a total order.
// ---------------------------------------------------------------------------
namespace {
// Memory-management kernel time attached to kernel k of tenant j (R31).
inline int64_t io_of(const Profile& prof, int j, int k) {
  const TenantProfile& tn = prof.ten[j];
  return (k == 0 ? tn.io_in : 0) + (k == (int)tn.k.size() - 1 ? tn.io_out : 0);
}

struct Order {
  int64_t now;
  const std::vector<int>* nxt;
  const std::vector<int64_t>* arr;
  const Profile* prof;
  int64_t tau(int j) const {
    int n = (*nxt)[j];
    return n == 0 ? 0 : prof->ten[j].tau_prog[n - 1];
  }
  bool more_behind(int x, int y) const {
    const int64_t tx = tau(x), ty = tau(y);
    if ((tx == 0) != (ty == 0)) return tx == 0;
    if (tx != 0) {
      const int64_t ex = std::max<int64_t>(0, now - (*arr)[x]);
      const int64_t ey = std::max<int64_t>(0, now - (*arr)[y]);
      const __int128 a = (__int128)ex * ty, b = (__int128)ey * tx;
      if (a != b) return a > b;
    }
    if (tx != ty) return tx < ty;
    if ((*arr)[x] != (*arr)[y]) return (*arr)[x] < (*arr)[y];
    return x < y;
  }
};
}  // namespace

void decide(int64_t now, const ActiveReq* act, int n_act, const Profile& prof, const SchedParams& prm,
            Decision& out, DecideScratch& sc) {
  const int nt = (int)prof.ten.size();
  const int S = prof.S, g = prof.g, N = prof.N;
  sc.nxt.assign(nt, -1);
  sc.arr.assign(nt, 0);
  out.active.clear();
  for (int i = 0; i < n_act; ++i) {
    sc.nxt[act[i].tenant] = act[i].next;
    sc.arr[act[i].tenant] = act[i].arrival;
  }
  for (int j = 0; j < nt; ++j)
    if (sc.nxt[j] >= 0) out.active.push_back({j, sc.arr[j], sc.nxt[j]});
  out.now = now;
  out.picks.clear();

  Order ord{now, &sc.nxt, &sc.arr, &prof};
  std::vector<int>& tenants = sc.order;
  tenants.clear();
  for (auto& a : out.active) tenants.push_back(a.tenant);

  // R36: a squad of a single active request closes after squad_max_solo
  // kernels (an arrival then waits at most that long for the next decision)
  const int cap = (out.active.size() == 1 && prm.squad_max_solo > 0) ? std::min(prm.squad_max, prm.squad_max_solo)
                                                                       : prm.squad_max;
  // §4.3.2 squad generation (L181-L187).
  auto pick = [&](int j) -> bool {
    const int k = sc.nxt[j];
    out.picks.push_back({j, k, 0, S});
    sc.nxt[j] = k + 1;
    return (int)out.picks.size() >= cap || k == (int)prof.ten[j].k.size() - 1;  // R5 / R36, R7
  };
  bool closed = false;
  if (prm.ablate & 1) {
    // §6.8 ablation (L426, R32): no multi-task scheduler -- one kernel per
    // active request per round in tenant-id order, same closing rules
    while (!closed) {
      for (int j : tenants)
        if (sc.nxt[j] < (int)prof.ten[j].k.size() && pick(j)) { closed = true; break; }
    }
  }
  if (!closed && prm.seed_all && tenants.size() >= 2) {  // R6
    std::vector<int> seed = tenants;
    std::sort(seed.begin(), seed.end(), [&](int x, int y) { return ord.more_behind(x, y); });
    for (int j : seed)
      if (pick(j)) { closed = true; break; }
  }
  while (!closed) {
    int best = -1;
    for (int j : tenants) {
      if (sc.nxt[j] >= (int)prof.ten[j].k.size()) continue;
      if (best < 0 || ord.more_behind(j, best)) best = j;
    }
    closed = pick(best);  // a request's last kernel always closes, so best >= 0
  }

  // Participants (sorted tenant ids) and their picks.
  out.parts.clear();
  for (auto& a : out.active)
    if (sc.nxt[a.tenant] > a.next) out.parts.push_back(a.tenant);
  const int K = (int)out.parts.size();
  if ((int)sc.ks.size() < K) sc.ks.resize(K);
  for (int i = 0; i < K; ++i) sc.ks[i].clear();
  {
    std::vector<int> slot(nt, -1);
    for (int i = 0; i < K; ++i) slot[out.parts[i]] = i;
    for (auto& pk : out.picks) sc.ks[slot[pk.tenant]].push_back(pk.kernel);
  }

  // Eq. 2 (L224, R12): NSP prediction over levels.
  int q = 0;
  for (int i = 0; i < K; ++i) q = std::max(q, (int)sc.ks[i].size());
  int64_t t_nsp = 0;
  std::vector<int64_t> level_end(q);
  for (int lv = 0; lv < q; ++lv) {
    int64_t x = 0;
    for (int i = 0; i < K; ++i)
      if ((int)sc.ks[i].size() > lv) x += prof.ten[out.parts[i]].k[sc.ks[i][lv]].d;
    x = std::min<int64_t>(x, S);
    int64_t level = 0;
    for (int i = 0; i < K; ++i) {
      if ((int)sc.ks[i].size() <= lv) continue;
      const int j = out.parts[i], k = sc.ks[i][lv];
      const int dk = prof.ten[j].k[k].d;
      if (x <= dk) level += prof.t(j, k, (int)x);
      else level += (prof.t(j, k, dk) * dk) / x;
      level += io_of(prof, j, k);   // R31
    }
    t_nsp += level;
    level_end[lv] = t_nsp;
  }
  out.t_nsp = t_nsp;
  out.t_hat = t_nsp;
  out.sp = false;
  out.p.clear();

  // Eq. 1 (L211) over all compositions by exact DP over suffixes (R9-R14);
  // skipped by the §6.8 ablation without the determiner (R32: always NSP).
  if (K >= 2 && !(prm.ablate & 2)) {
    const int W = N + 1;
    sc.Sj.assign((size_t)K * W, 0);
    sc.F.assign((size_t)K * W, INT64_MAX);
    for (int i = 0; i < K; ++i) {
      const int j = out.parts[i];
      for (int p = 1; p <= N; ++p) {
        const int s = (i < K - 1) ? g * p : S - g * (N - p);
        int64_t sum = 0;
        for (int k : sc.ks[i]) sum += prof.t(j, k, s) + io_of(prof, j, k);   // R31
        sc.Sj[(size_t)i * W + p] = sum;
      }
    }
    // F[K-1][r] = chain of the last participant with r partitions.
    for (int r = 1; r <= N; ++r) sc.F[(size_t)(K - 1) * W + r] = sc.Sj[(size_t)(K - 1) * W + r];
    for (int i = K - 2; i >= 0; --i) {
      const int rest = K - 1 - i;  // participants after i, each needs >= 1
      for (int r = rest + 1; r <= N; ++r) {
        int64_t best = INT64_MAX;
        for (int p = 1; p <= r - rest; ++p) {
          const int64_t v = std::max(sc.Sj[(size_t)i * W + p], sc.F[(size_t)(i + 1) * W + (r - p)]);
          if (v < best) best = v;
        }
        sc.F[(size_t)i * W + r] = best;
      }
    }
    const int64_t opt = sc.F[N];  // F[0][N]
    if (opt < t_nsp) {            // R13: strictly better than NSP
      out.sp = true;
      out.t_hat = opt;
      out.p.assign(K, 0);
      int r = N;
      for (int i = 0; i < K - 1; ++i) {  // R14: lexicographically smallest optimum
        const int rest = K - 1 - i;
        for (int p = 1; p <= r - rest; ++p) {
          const int64_t v = std::max(sc.Sj[(size_t)i * W + p], sc.F[(size_t)(i + 1) * W + (r - p)]);
          if (v <= opt) { out.p[i] = p; break; }
        }
        r -= out.p[i];
      }
      out.p[K - 1] = r;
    }
  }

  // Predicted end of each participant's picks (for the model clock / logs).
  out.chain_end.assign(K, 0);
  if (out.sp) {
    const int W = N + 1;
    for (int i = 0; i < K; ++i) out.chain_end[i] = sc.Sj[(size_t)i * W + out.p[i]];
  } else {
    for (int i = 0; i < K; ++i) out.chain_end[i] = level_end[sc.ks[i].size() - 1];
  }

  // Semi-SP range plan (L253-L255, R16).
  if (out.sp) {
    std::vector<int> lo(nt, 0), hi(nt, S), rcount(nt, 0), seen(nt, 0);
    int base = 0;
    for (int i = 0; i < K; ++i) {
      const int j = out.parts[i];
      lo[j] = base;
      hi[j] = (i == K - 1) ? S : base + g * out.p[i];
      base = hi[j];
      rcount[j] = ((int)sc.ks[i].size() * prm.split_pct + 99) / 100;
    }
    for (auto& pk : out.picks) {
      if (seen[pk.tenant] < rcount[pk.tenant]) { pk.lo = lo[pk.tenant]; pk.hi = hi[pk.tenant]; }
      seen[pk.tenant] += 1;
    }
  }
}

// Eq. 2 (L224, R12) for a given squad: levels i = 0..q-1, x_i = min(S, sum of
// d over the level), work-equivalent time t[d]*d/x past a kernel's d (same
// arithmetic as decide()).
int64_t predict_nsp(const Profile& prof, const std::vector<int>& parts, const std::vector<std::vector<int>>& ks) {
  const int K = (int)parts.size(), S = prof.S;
  int q = 0;
  for (int i = 0; i < K; ++i) q = std::max(q, (int)ks[i].size());
  int64_t t = 0;
  for (int lv = 0; lv < q; ++lv) {
    int64_t x = 0;
    for (int i = 0; i < K; ++i)
      if ((int)ks[i].size() > lv) x += prof.ten[parts[i]].k[ks[i][lv]].d;
    x = std::min<int64_t>(x, S);
    for (int i = 0; i < K; ++i) {
      if ((int)ks[i].size() <= lv) continue;
      const int j = parts[i], k = ks[i][lv];
      const int dk = prof.ten[j].k[k].d;
      t += (x <= dk) ? prof.t(j, k, (int)x) : (prof.t(j, k, dk) * dk) / x;
      t += io_of(prof, j, k);
    }
  }
  return t;
}

// Eq. 1 (L211) for a given composition p of N partitions (R9-R11): the
// slowest participant chain on its g*p_i SMs (the last one gets the rest).
int64_t predict_sp(const Profile& prof, const std::vector<int>& parts, const std::vector<std::vector<int>>& ks,
                   const std::vector<int>& p) {
  const int K = (int)parts.size(), S = prof.S, g = prof.g, N = prof.N;
  int64_t worst = 0;
  for (int i = 0; i < K; ++i) {
    const int s = (i < K - 1) ? g * p[i] : S - g * (N - p[i]);
    int64_t sum = 0;
    for (int k : ks[i]) sum += prof.t(parts[i], k, s) + io_of(prof, parts[i], k);
    worst = std::max(worst, sum);
  }
  return worst;
}

bool colocatable(const std::vector<int64_t>& avg, int64_t span_x) {
  if (avg.empty()) return true;
  const int64_t lo = *std::min_element(avg.begin(), avg.end());
  const int64_t hi = *std::max_element(avg.begin(), avg.end());
  return (__int128)hi <= (__int128)lo * span_x;   // exact: max <= span * min
}

std::vector<int> place(const std::vector<int64_t>& mem, const std::vector<int64_t>& avg,
                       const std::vector<int64_t>& gpu_free, int64_t span_x) {
  const int n = (int)mem.size(), G = (int)gpu_free.size();
  std::vector<int> order(n), out(n, -1);
  for (int i = 0; i < n; ++i) order[i] = i;
  std::stable_sort(order.begin(), order.end(), [&](int a, int b) { return mem[a] > mem[b]; });
  std::vector<int64_t> left = gpu_free;
  std::vector<std::vector<int64_t>> on(G);
  for (int a : order) {
    int best = -1;
    for (int gpu = 0; gpu < G; ++gpu) {
      if (mem[a] > left[gpu]) continue;
      std::vector<int64_t> v = on[gpu];
      v.push_back(avg[a]);
      if (!colocatable(v, span_x)) continue;
      if (best < 0 || left[gpu] > left[best]) best = gpu;
    }
    if (best >= 0) {
      out[a] = best;
      left[best] -= mem[a];
      on[best].push_back(avg[a]);
    }
  }
  return out;
}

}  // namespace bless
