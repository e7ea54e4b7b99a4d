// capi.cpp -- extern "C" boundary (include/bless/bless.h).  Argument checks,
// error strings and exception containment only; all logic is in Engine.
#include <chrono>
#include <exception>
#include <string>

#include "../../include/bless/bless.h"
#include "runtime/engine.hpp"

struct bl_ctx {
  bless::Engine* eng;
};

static thread_local std::string g_err;

#define GUARD(ctx)                                      \
  if (!(ctx) || !(ctx)->eng) {                          \
    g_err = "null ctx";                                 \
    return BL_E_INVALID;                                \
  }

template <class F>
static bl_status wrap(F&& f) {
  try {
    std::string err;
    bl_status st = f(err);
    if (st != BL_OK && st != BL_PENDING) g_err = err;
    return st;
  } catch (const std::bad_alloc&) {
    g_err = "out of host memory";
    return BL_E_OOM;
  } catch (const std::exception& e) {
    g_err = e.what();
    return BL_E_INVALID;
  } catch (...) {
    g_err = "unknown exception";
    return BL_E_INVALID;
  }
}

extern "C" {

void bl_params_default(bl_params* p) {
  if (!p) return;
  *p = bl_params{};
  p->sm_unit = 4;
  p->squad_max = 50;
  p->split_pct = 50;
  p->seed_all = 1;
  p->policy = BL_POLICY_BLESS;
  p->clock = BL_CLOCK_WALL;
  p->squad_overhead_ns = 0;
  p->temporal_period_ns = 2000000;
  p->temporal_work_conserving = 0;
  p->max_inflight_squads = 2;
  p->lookahead_ns = 20000;
  p->max_requests = 1 << 20;
  p->squad_max_solo = 0;
}

bl_status bl_create(int device, const bl_params* params, void* ws, size_t ws_bytes, bl_ctx** out) {
  if (!out) { g_err = "null out"; return BL_E_INVALID; }
  *out = nullptr;
  bl_params p;
  bl_params_default(&p);
  if (params) p = *params;
  return wrap([&](std::string& err) {
    bless::Engine* e = new bless::Engine(device, p);
    bl_status st = e->init(ws, ws_bytes, err);
    if (st != BL_OK) { delete e; return st; }
    *out = new bl_ctx{e};
    return BL_OK;
  });
}

bl_status bl_destroy(bl_ctx* ctx) {
  GUARD(ctx);
  delete ctx->eng;
  ctx->eng = nullptr;
  delete ctx;
  return BL_OK;
}

bl_status bl_device_info_get(bl_ctx* ctx, bl_device_info* out) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->device_info(out, e); });
}
bl_status bl_register_tenant(bl_ctx* ctx, double quota, const char* name, int* tenant_out) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->register_tenant(quota, name, tenant_out, e); });
}
bl_status bl_set_tenant_slo(bl_ctx* ctx, int tenant, int64_t slo_ns) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->set_slo(tenant, slo_ns, e); });
}
bl_status bl_set_stream(bl_ctx* ctx, int tenant, void* s) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->set_stream(tenant, s, e); });
}
bl_status bl_append_kernel(bl_ctx* ctx, int tenant, const bl_op* op, int* k) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->append_kernel(tenant, op, k, e); });
}
bl_status bl_run_kernel(bl_ctx* ctx, int tenant, int k, int lo, int hi) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->run_kernel(tenant, k, lo, hi, e); });
}
bl_status bl_set_tenant_io(bl_ctx* ctx, int tenant, const void* hin, void* din, size_t inb, const void* dout,
                           void* hout, size_t outb) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->set_io(tenant, hin, din, inb, dout, hout, outb, e); });
}
bl_status bl_kernel_info_get(bl_ctx* ctx, int tenant, int k, bl_kernel_info* out) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->kernel_info(tenant, k, out, e); });
}
bl_status bl_profile_kernel(bl_ctx* ctx, int tenant, int k, int sm_count, int reps, int64_t* ns, int* d) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->profile_kernel(tenant, k, sm_count, reps, ns, d, e); });
}
bl_status bl_profile_tenant(bl_ctx* ctx, int tenant, int reps) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->profile_tenant(tenant, reps, e); });
}
bl_status bl_set_profile_row(bl_ctx* ctx, int tenant, int k, const int64_t* t, int d) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->set_profile_row(tenant, k, t, d, e); });
}
bl_status bl_get_profile_row(bl_ctx* ctx, int tenant, int k, int64_t* t, int* d) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->get_profile_row(tenant, k, t, d, e); });
}
bl_status bl_save_profile(bl_ctx* ctx, const char* path) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->save_profile(path, e); });
}
bl_status bl_load_profile(bl_ctx* ctx, const char* path) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->load_profile(path, e); });
}
bl_status bl_tenant_info(bl_ctx* ctx, int tenant, int* qsms, int* m, int64_t* T) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->tenant_info(tenant, qsms, m, T, e); });
}
bl_status bl_start(bl_ctx* ctx) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->start(e); });
}
bl_status bl_submit(bl_ctx* ctx, int tenant, int64_t arrival_ns, uint64_t* req_out) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->submit(tenant, arrival_ns, req_out, e); });
}
bl_status bl_poll(bl_ctx* ctx, uint64_t req, bl_req_info* out) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->poll(req, out, e); });
}
bl_status bl_drain(bl_ctx* ctx, int64_t timeout_ns) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->drain(timeout_ns, e); });
}
bl_status bl_stop(bl_ctx* ctx) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->stop(e); });
}
bl_status bl_decisions(bl_ctx* ctx, size_t first, bl_decision* buf, size_t cap, size_t* n) {
  GUARD(ctx);
  return ctx->eng->decisions(first, buf, cap, n);
}
bl_status bl_launches(bl_ctx* ctx, size_t first, bl_launch_rec* buf, size_t cap, size_t* n) {
  GUARD(ctx);
  return ctx->eng->launches(first, buf, cap, n);
}
bl_status bl_temporal_log(bl_ctx* ctx, size_t first, bl_temporal_rec* buf, size_t cap, size_t* n) {
  GUARD(ctx);
  return ctx->eng->temporal_log(first, buf, cap, n);
}
bl_status bl_time_decide(bl_ctx* ctx, const bl_decision* recs, size_t n, int reps, int64_t* total_ns,
                         int64_t* total_picks) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->time_decide(recs, n, reps, total_ns, total_picks, e); });
}
bl_status bl_dispatch(bl_ctx* const* ctxs, int n_ctx, const bl_dispatch_entry* ent, size_t n, int64_t base_ns,
                      uint64_t* req_out) {
  if (!ctxs || n_ctx < 1 || (n && !ent)) {
    g_err = "bad dispatcher args";
    return BL_E_INVALID;
  }
  for (int i = 0; i < n_ctx; ++i) GUARD(ctxs[i]);
  return wrap([&](std::string& e) {
    int64_t prev = INT64_MIN;
    for (size_t i = 0; i < n; ++i) {
      const bl_dispatch_entry& x = ent[i];
      if (x.ctx < 0 || x.ctx >= n_ctx) { e = "entry " + std::to_string(i) + ": bad ctx index"; return BL_E_INVALID; }
      if (x.arrival_ns < prev) { e = "entries not sorted by arrival"; return BL_E_INVALID; }
      prev = x.arrival_ns;
      bless::Engine* eng = ctxs[x.ctx]->eng;
      int64_t arr = x.arrival_ns;
      if (!eng->virtual_clock()) {
        // a steady-clock busy-wait: the request is handed over at its arrival
        arr = base_ns + x.arrival_ns;
        while (bl_now_ns() < arr) {
#if defined(__x86_64__)
          __builtin_ia32_pause();
#endif
        }
      }
      uint64_t id = 0;
      const bl_status st = eng->submit(x.tenant, arr, &id, e);
      if (st != BL_OK) return st;
      if (req_out) req_out[i] = id;
    }
    return BL_OK;
  });
}
bl_status bl_predict(bl_ctx* ctx, int n, const int32_t* ten, const int32_t* ker, const int32_t* p, int64_t* out) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->predict(n, ten, ker, p, out, e); });
}
bl_status bl_run_squad(bl_ctx* ctx, int n, const int32_t* ten, const int32_t* ker, const int16_t* lo,
                       const int16_t* hi, int reps, int64_t* makespan, int64_t* kernel_ns) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->run_squad(n, ten, ker, lo, hi, reps, makespan, kernel_ns, e); });
}
bl_status bl_deployment_check(bl_ctx* ctx, const int64_t* mem, int64_t free_b, int32_t span, int32_t* ok,
                              int32_t* why) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->deployment_check(mem, free_b, span, ok, why, e); });
}
bl_status bl_place(int n, const int64_t* mem, const int64_t* avg, int G, const int64_t* gfree, int32_t span,
                   int32_t* out) {
  if (n < 0 || G < 1 || span < 1 || (n && (!mem || !avg || !out)) || !gfree) {
    g_err = "bad placement args";
    return BL_E_INVALID;
  }
  return wrap([&](std::string&) {
    const std::vector<int> r = bless::place(std::vector<int64_t>(mem, mem + n), std::vector<int64_t>(avg, avg + n),
                                            std::vector<int64_t>(gfree, gfree + G), span);
    for (int i = 0; i < n; ++i) out[i] = r[i];
    return BL_OK;
  });
}
bl_status bl_reset(bl_ctx* ctx, const bl_params* p) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->reset(p, e); });
}
bl_status bl_decide(bl_ctx* ctx, int64_t now, int n, const int32_t* t, const int64_t* a, const int32_t* k,
                    bl_decision* out) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->decide_pure(now, n, t, a, k, out, e); });
}

bl_status bl_debug_overhead(bl_ctx* ctx, int variant, int reps, int64_t* ns) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->debug_overhead(variant, reps, ns, e); });
}

bl_status bl_debug_chain(bl_ctx* ctx, int tenant, int lo, int hi, int graph, int reps, int64_t* device_ns,
                         int64_t* host_ns) {
  GUARD(ctx);
  return wrap([&](std::string& e) { return ctx->eng->debug_chain(tenant, lo, hi, graph, reps, device_ns, host_ns, e); });
}

int64_t bl_now_ns(void) {
  return std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now().time_since_epoch())
      .count();
}
const char* bl_last_error(void) { return g_err.c_str(); }
const char* bl_version(void) { return "blessb200 0.1 (sm_100a)"; }

}  // extern "C"
