"""Evaluation sweeps of SURVEY.md §8(f) f4 on one B200 (§6.4, §6.7,
§4.2.2):

* multiapp -- more than two co-located applications whose requests arrive at
  the same time (L354-L360, Table 2): identical ResNet50 tenants with the
  4-model quotas (10, 20, 30, 40%) and the 8-model quotas (5, 5, 10, 10, 15,
  15, 20, 20%).  Paper (A100): 4 apps -41.2% / -18.3% vs TEMPORAL / GSLICE;
  8 apps -80.8% / -35.5%, latency deviation BLESS 0, TEMPORAL 74 ms, GSLICE
  5 ms, UNBOUND 3.8 ms.
* smsweep  -- the SM-count sweep (L420): two symmetric ResNet50 tenants (1/2
  each) under low load (workload C), the whole system restricted to the first
  s SMs (bl_params.sm_limit, the way the paper restricts the GPU with MIG);
  BLESS's latency reduction vs the static split (GSLICE analog) per s.  Paper:
  54.4% -> 40.2% as the SM count grows.
* deploy   -- deployment admission (L163-L169) and placement (L171) over our
  nine tenant models with their profiled average kernel durations and their
  device memory (reading R33).

  python tools/f4_sweeps.py multiapp|smsweep|deploy [--out gpurun_out/f4_x.json]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

POLICIES = [("BLESS", {}), ("STATIC", {}), ("TEMPORAL_Tcap", {"policy": "TEMPORAL"}),
            ("TEMPORAL_Twc", {"policy": "TEMPORAL", "temporal_work_conserving": 1}), ("UNBOUND", {})]


def build_tenants(ctx, models, names, quotas):
    ms = []
    for i, (n, q) in enumerate(zip(names, quotas)):
        t = ctx.register_tenant(q, f"{n}{i}")
        ms.append(models.BUILDERS[n](ctx, t, q, dtype="bf16", seed=1000 + i))
    return ms


def run(ctx, capi, params, entries, nt, only=None):
    ctx.reset(params)
    ctx.start()
    ents = [e for e in entries if only is None or e[1] in only]
    ids = capi.dispatch([ctx], ents, capi.now_ns() + 3_000_000)
    ctx.drain(int(300e9))
    ctx.stop()
    lat = {j: [] for j in range(nt)}
    for (_, t, _), r in zip(ents, ids):
        st, info = ctx.poll(r)
        assert st == capi.BL_OK
        lat[t].append(info.finish_ns - info.arrival_ns)
    return lat


def policy_table(ctx, capi, metrics, entries, nt, squad_max, extra=None):
    out = {}
    means = {}
    for label, kw in POLICIES:
        kw = dict(kw)
        pol = kw.pop("policy", label)
        p = capi.default_params(policy=pol, squad_max=squad_max, split_pct=25, **kw, **(extra or {}))
        lat = run(ctx, capi, p, entries, nt)
        means[label] = {j: float(np.mean(v)) for j, v in lat.items()}
        out[label] = float(np.mean([x for v in lat.values() for x in v])) / 1e6
    iso = {}
    for j in range(nt):
        p = capi.default_params(policy="ISO", squad_max=squad_max, **(extra or {}))
        iso[j] = float(np.mean(run(ctx, capi, p, entries, nt, {j})[j]))
    dev = {k: metrics.latency_deviation(v, iso) / 1e6 for k, v in means.items()}
    att = {j: metrics.attainment_pct(iso[j], means["BLESS"][j]) for j in range(nt)}
    return {"mean_ms": out, "iso_mean_ms": {j: v / 1e6 for j, v in iso.items()}, "deviation_ms": dev,
            "bless_attainment_pct": att,
            "bless_vs_temporal_tcap_pct": 100 * (out["BLESS"] / out["TEMPORAL_Tcap"] - 1),
            "bless_vs_temporal_twc_pct": 100 * (out["BLESS"] / out["TEMPORAL_Twc"] - 1),
            "bless_vs_static_pct": 100 * (out["BLESS"] / out["STATIC"] - 1),
            "bless_vs_unbound_pct": 100 * (out["BLESS"] / out["UNBOUND"] - 1)}


def multiapp(a, capi, models, metrics):
    from synth import trace as tr
    res = {}
    for label, quotas in (("4 apps (10/20/30/40%)", [0.1, 0.2, 0.3, 0.4]),
                          ("8 apps (5/5/10/10/15/15/20/20%)", [0.05, 0.05, 0.1, 0.1, 0.15, 0.15, 0.2, 0.2])):
        ctx = capi.Ctx(0, squad_max=20)
        ms = build_tenants(ctx, models, ["resnet50"] * len(quotas), quotas)
        for m in ms:
            ctx.profile_tenant(m.tenant, reps=3)
        T = [ctx.tenant_info(m.tenant)[2] for m in ms]
        # all applications' requests arrive at the same time (L356), one round
        # every 1.5 x the slowest isolated latency
        trace = tr.simultaneous(len(ms), a.rounds, int(1.5 * max(T)))
        ents = [(0, x.tenant, x.arrival_ns) for x in trace]
        row = policy_table(ctx, capi, metrics, ents, len(ms), 20)
        row["quota_sms"] = [ctx.tenant_info(m.tenant)[0] for m in ms]
        row["T_iso_profile_ms"] = [t / 1e6 for t in T]
        res[label] = row
        print(label, json.dumps(row), flush=True)
        ctx.close()
    res["paper"] = {"4 apps": {"vs_temporal_pct": -41.2, "vs_gslice_pct": -18.3},
                    "8 apps": {"vs_temporal_pct": -80.8, "vs_gslice_pct": -35.5,
                               "deviation_ms": {"BLESS": 0, "TEMPORAL": 74, "GSLICE": 5, "UNBOUND": 3.8}}}
    return res


def smsweep(a, capi, models, metrics):
    from synth import trace as tr
    ctx = capi.Ctx(0, squad_max=20)
    ms = build_tenants(ctx, models, ["resnet50", "resnet50"], [0.5, 0.5])
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=3)
    S = ctx.device_info().sm_count
    res = {}
    for s in a.sms:
        s = min(s, S)
        # profile-derived T at the restricted quota: run an ISO pass to learn it
        p = capi.default_params(policy="BLESS", squad_max=20, sm_limit=s)
        ctx.reset(p)
        ctx.start()
        T = [ctx.tenant_info(m.tenant)[2] for m in ms]
        ctx.stop()
        trace = tr.poisson([t / a.rho for t in T], a.requests, seed=3)
        ents = [(0, x.tenant, x.arrival_ns) for x in trace]
        row = policy_table(ctx, capi, metrics, ents, 2, 20, {"sm_limit": s})
        row["sm_limit"] = s
        res[str(s)] = row
        print(f"S={s}", json.dumps(row), flush=True)
    ctx.close()
    res["paper"] = {"bless_vs_gslice_reduction_pct": "54.4 -> 40.2 as SMs grow (A100 MIG slices)"}
    return res


def deploy(a, capi, models, metrics):
    import torch
    rows = {}
    S = None
    for cfg, spec in models.CONFIGS.items():
        if cfg == "C1":
            continue
        ctx = capi.Ctx(0)
        S = ctx.device_info().sm_count
        ms = models.build_config(ctx, cfg, "bf16")
        for m in ms:
            ctx.profile_tenant(m.tenant, reps=2)
        mem = [int(sum(t.numel() * t.element_size() for t in m.keep)) for m in ms]
        ok, why = ctx.deployment_check(mem, 0, 30)
        info = []
        for m, mb in zip(ms, mem):
            q, n, T = ctx.tenant_info(m.tenant)
            info.append({"tenant": m.name, "quota_sms": q, "kernels": n, "T_iso_us": T / 1e3,
                         "avg_kernel_us": T / n / 1e3, "mem_mb": mb / 2**20})
        rows[cfg] = {"tenants": info, "admissible_span30": ok, "reason": why,
                     "admissible_span5": ctx.deployment_check(mem, 0, 5)[0]}
        print(cfg, json.dumps(rows[cfg]), flush=True)
        ctx.close()
        torch.cuda.empty_cache()
    # central-controller placement of all nine models onto an 8-GPU box (L171)
    apps = [t for r in rows.values() for t in r["tenants"]]
    mem = [int(t["mem_mb"] * 2**20) for t in apps]
    avg = [int(t["avg_kernel_us"] * 1e3) for t in apps]
    free = [int(170e9)] * 8
    rows["placement_8gpu"] = {"apps": [t["tenant"] for t in apps],
                              "gpu_span30": capi.place(mem, avg, free, 30),
                              "gpu_span5": capi.place(mem, avg, free, 5),
                              "gpu_span5_2gpu_2GB": capi.place(mem, avg, [2 << 30] * 2, 5)}
    print(json.dumps(rows["placement_8gpu"]), flush=True)
    return rows


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("what", choices=["multiapp", "smsweep", "deploy"])
    ap.add_argument("--rounds", type=int, default=12)
    ap.add_argument("--rho", type=float, default=0.3)
    ap.add_argument("--requests", type=int, default=60)
    ap.add_argument("--sms", type=lambda s: [int(x) for x in s.split(",")], default=[36, 72, 108, 148])
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi, metrics, models
    build.build(verbose=False)
    res = {"multiapp": multiapp, "smsweep": smsweep, "deploy": deploy}[a.what](a, capi, models, metrics)
    if a.out:
        os.makedirs(os.path.dirname(os.path.abspath(a.out)), exist_ok=True)
        json.dump(res, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
