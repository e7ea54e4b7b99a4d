"""Per-tenant request latency breakdown under BLESS vs ISO / STATIC / UNBOUND
on the same traces (C2 by default): queueing (arrival -> first kernel start)
and service (first kernel start -> completion), plus how BLESS's squads mix
the tenants.  Explains quota attainment.

  python tools/breakdown.py [--config C2] [--rho 0.5] [--requests 100]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--rho", type=float, default=0.5)
    ap.add_argument("--requests", type=int, default=100)
    ap.add_argument("--squad-max", type=int, default=20)
    ap.add_argument("--split-pct", type=int, default=25)
    ap.add_argument("--max-inflight", type=int, default=2)
    ap.add_argument("--squad-max-solo", type=int, default=0)
    ap.add_argument("--lookahead-us", type=float, default=20.0)
    ap.add_argument("--barrier", type=int, default=0)
    ap.add_argument("--policies", default="BLESS,ISO,STATIC,UNBOUND")
    a = ap.parse_args()
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi, models
    from synth import trace as tr
    build.build(verbose=False)
    ctx = capi.Ctx(0)
    ms = models.build_config(ctx, a.config, "bf16")
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=5)
    T = [ctx.tenant_info(m.tenant)[2] for m in ms]
    out = {}
    for seed in (1, 2, 3):
        trace = tr.poisson([t / a.rho for t in T], a.requests, seed=seed)
        for pol in a.policies.split(","):
            filts = [{j} for j in range(len(ms))] if pol == "ISO" else [None]
            for filt in filts:
                p = capi.default_params(policy=pol, squad_max=a.squad_max, split_pct=a.split_pct,
                                        max_inflight_squads=a.max_inflight, lookahead_ns=int(a.lookahead_us * 1000),
                                        squad_max_solo=a.squad_max_solo, barrier=a.barrier)
                ctx.reset(p)
                ctx.start()
                ents = [(0, x.tenant, x.arrival_ns) for x in trace if filt is None or x.tenant in filt]
                ids = capi.dispatch([ctx], ents, capi.now_ns() + 3_000_000)
                ctx.drain(int(120e9))
                ctx.stop()
                infos = []
                for (_, t, _), r in zip(ents, ids):
                    st, info = ctx.poll(r)
                    infos.append((t, info.arrival_ns, info.start_ns, info.finish_ns))
                    d = out.setdefault(pol, {}).setdefault(ms[t].name, {"wait": [], "service": [], "lat": []})
                    d["wait"].append(info.start_ns - info.arrival_ns)
                    d["service"].append(info.finish_ns - info.start_ns)
                    d["lat"].append(info.finish_ns - info.arrival_ns)
                if filt is None:
                    # wait split by what the GPU was doing at the arrival: another
                    # tenant's request in progress or not; own previous request
                    # still in progress (FIFO) or not
                    for t, arr, s0, _f in infos:
                        other = any(t2 != t and a2 <= arr < f2 for t2, a2, _, f2 in infos)
                        own = any(t2 == t and a2 < arr < f2 for t2, a2, _, f2 in infos)
                        key = ("other_busy" if other else "other_idle") + ("+own_queue" if own else "")
                        ws = out.setdefault(pol + "_wait_by_state", {}).setdefault(ms[t].name, {}).setdefault(key, [])
                        ws.append(s0 - arr)
                if pol == "BLESS":
                    decs = [capi.decision_to_tuple(x) for x in ctx.decisions()]
                    mix = out.setdefault("squads", {"solo": 0, "mixed_nsp": 0, "mixed_sp": 0})
                    for dd in decs:
                        if len(dd["parts"]) == 1:
                            mix["solo"] += 1
                        elif dd["config"] is None:
                            mix["mixed_nsp"] += 1
                        else:
                            mix["mixed_sp"] += 1
    summ = {}
    for pol, per in out.items():
        if pol == "squads":
            summ[pol] = per
            continue
        if pol.endswith("_wait_by_state"):
            summ[pol] = {n: {k: {"n": len(v), "mean_us": float(np.mean(v)) / 1e3} for k, v in d.items()}
                         for n, d in per.items()}
            continue
        summ[pol] = {n: {k: float(np.mean(v)) / 1e3 for k, v in d.items()} for n, d in per.items()}
    print(json.dumps(summ, indent=1))
    ctx.close()


if __name__ == "__main__":
    main()
