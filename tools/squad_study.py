"""Predictor accuracy and squad-mode study on B200.

The paper measures, on A100: the interference-free predictor Eq. 1 at 6.7%
error and the workload-equivalence predictor Eq. 2 at 7.1% (L214, L227); the
predicted configuration equal to the real optimum in 96.2% of 2,260 kernel
groups (L237); kernel slowdowns from interference up to 2x, 7% at application
level (L218-L220); and squad duration against sequential execution: NSP
-6.5%, SP -12.9%, Semi-SP -17.6% (L382; Fig. 7 / Fig. 17).

This tool repeats the study on our kernels.  It profiles a config, runs BLESS
on a Poisson trace to collect real kernel squads with >= 2 participants,
samples them, and executes each sampled squad on the GPU (bl_run_squad) as:

* NSP  -- every pick on all S SMs (Eq. 2 predicts it);
* SP   -- every pick of participant i on its own window of a split p
          (Eq. 1 predicts it): all C(N-1, 1) splits for K = 2, otherwise
          the Eq. 1 optimum plus random splits;
* Semi-SP -- the split and c% ranges BLESS chose (L253-L255);
* SEQ  -- each participant's picks alone on all S SMs, one after the other.

It reports the mean absolute error of Eq. 1 / Eq. 2 against the measured
makespans, how often the predicted-best configuration (over the evaluated
set) is the measured best (exactly, and within 2%), each mode's squad
duration relative to SEQ, and the per-kernel interference slowdown
(duration inside the squad / isolated profile at the same SM count).

  python tools/squad_study.py --config C2 --squads 40 --out gpurun_out/f1_c2.json
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def compositions(N, K):
    if K == 1:
        yield (N,)
        return
    for first in range(1, N - K + 2):
        for rest in compositions(N - first, K - 1):
            yield (first,) + rest


def windows(p, S, g):
    out, lo = [], 0
    for i, x in enumerate(p):
        hi = S if i == len(p) - 1 else lo + g * x
        out.append((lo, hi))
        lo = hi
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--squads", type=int, default=40)
    ap.add_argument("--rho", type=float, default=0.5)
    ap.add_argument("--requests", type=int, default=40)
    ap.add_argument("--squad-max", type=int, default=0)
    ap.add_argument("--split-pct", type=int, default=25)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--random-splits", type=int, default=12)
    ap.add_argument("--seed", type=int, default=5)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "squad_study.json"))
    a = ap.parse_args()
    import torch

    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi, models
    from synth import trace as tr
    build.build(verbose=False)
    smax = a.squad_max or {"C1": 4, "C2": 20, "C3": 10, "C4": 10}[a.config]
    ctx = capi.Ctx(0, squad_max=smax, split_pct=a.split_pct)
    S = ctx.device_info().sm_count
    g = ctx.params.sm_unit
    N = S // g
    ms = models.build_config(ctx, a.config, "fp32" if a.config == "C1" else "bf16")
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=5)
    prof_rows = {(m.tenant, k): ctx.get_profile_row(m.tenant, k, S)[0] for m in ms for k in range(len(m.layers))}
    T = [ctx.tenant_info(m.tenant)[2] for m in ms]
    trace = tr.poisson([t / a.rho for t in T], a.requests, seed=a.seed)
    ctx.start()
    base = capi.now_ns() + 2_000_000
    for x in trace:
        ctx.submit(x.tenant, base + x.arrival_ns)
    ctx.drain(int(120e9))
    ctx.stop()
    decs = [capi.decision_to_tuple(d) for d in ctx.decisions()]
    cand = {}
    for d in decs:
        if len(d["parts"]) >= 2:
            cand.setdefault(tuple((t, k) for t, k, _, _ in d["picks"]), d)
    keys = sorted(cand)
    rng = np.random.Generator(np.random.PCG64(a.seed))
    sel = [keys[i] for i in sorted(rng.choice(len(keys), size=min(a.squads, len(keys)), replace=False))]

    rows = []
    for key in sel:
        d = cand[key]
        picks = list(key)
        parts = sorted({t for t, _ in picks})
        K = len(parts)
        res = {"picks": len(picks), "K": K, "tenants": parts, "bless_config": d["config"]}
        full = [(t, k, 0, S) for t, k in picks]
        nsp_ms, nsp_k = ctx.run_squad(full, a.reps)
        res["nsp"] = {"meas": nsp_ms, "pred": ctx.predict(picks)}
        seq = 0
        for j in parts:
            mine = [(t, k, 0, S) for t, k in picks if t == j]
            seq += ctx.run_squad(mine, a.reps)[0]
        res["seq"] = seq
        comps = list(compositions(N, K))
        if K == 2:
            evald = comps
        else:
            best = min(comps, key=lambda p: ctx.predict(picks, list(p)))
            extra = [comps[int(i)] for i in rng.choice(len(comps), size=min(a.random_splits, len(comps)),
                                                          replace=False)]
            evald = sorted(set([best] + extra + ([tuple(d["config"])] if d["config"] else [])))
        sp = []
        for p in evald:
            win = windows(p, S, g)
            widx = {j: win[i] for i, j in enumerate(parts)}
            run = [(t, k, *widx[t]) for t, k in picks]
            m_ns, k_ns = ctx.run_squad(run, a.reps)
            sp.append({"p": list(p), "meas": m_ns, "pred": ctx.predict(picks, list(p)),
                       "slow": [kn / max(1, prof_rows[(t, k)][widx[t][1] - widx[t][0] - 1])
                                for (t, k), kn in zip(picks, k_ns)]})
        res["sp"] = sp
        res["nsp"]["slow"] = [kn / max(1, prof_rows[(t, k)][S - 1]) for (t, k), kn in zip(picks, nsp_k)]
        if d["config"] is not None:
            semi = [(t, k, lo, hi) for t, k, lo, hi in d["picks"]]
            res["semi_sp"] = {"meas": ctx.run_squad(semi, a.reps)[0], "pred_eq1": d["t_hat"]}
        # best configuration over the evaluated set: predicted vs measured
        allc = [("NSP", res["nsp"]["pred"], res["nsp"]["meas"])] + [(tuple(x["p"]), x["pred"], x["meas"]) for x in sp]
        pb = min(allc, key=lambda c: (c[1], 0 if c[0] == "NSP" else 1, c[0] if c[0] != "NSP" else ()))
        mb = min(allc, key=lambda c: c[2])
        res["pred_best"], res["meas_best"] = str(pb[0]), str(mb[0])
        res["match_exact"] = pb[0] == mb[0]
        res["match_2pct"] = pb[2] <= 1.02 * mb[2]
        rows.append(res)
        print(f"squad K={K} picks={len(picks)}: NSP {nsp_ms / 1e3:.1f}us (pred {res['nsp']['pred'] / 1e3:.1f}) "
              f"SEQ {seq / 1e3:.1f}us  best SP {min(x['meas'] for x in sp) / 1e3:.1f}us "
              f"semi {res.get('semi_sp', {}).get('meas', 0) / 1e3:.1f}us  pred-best {res['pred_best']} "
              f"meas-best {res['meas_best']}", flush=True)

    def mape(pairs):
        v = [abs(m - p) / m for p, m in pairs if m > 0]
        return 100 * float(np.mean(v)) if v else None

    def bias(pairs):
        v = [(m - p) / m for p, m in pairs if m > 0]
        return 100 * float(np.mean(v)) if v else None
    eq2 = [(r["nsp"]["pred"], r["nsp"]["meas"]) for r in rows]
    eq1 = [(x["pred"], x["meas"]) for r in rows for x in r["sp"]]
    eq1_best = [(min(r["sp"], key=lambda x: x["pred"])["pred"], min(r["sp"], key=lambda x: x["pred"])["meas"])
                for r in rows]
    slow_nsp = [s for r in rows for s in r["nsp"]["slow"]]
    slow_sp = [s for r in rows for x in r["sp"] for s in x["slow"]]
    vs_seq = {"NSP": [r["nsp"]["meas"] / r["seq"] - 1 for r in rows],
              "SP_best": [min(x["meas"] for x in r["sp"]) / r["seq"] - 1 for r in rows],
              "SP_pred_best": [min(r["sp"], key=lambda x: x["pred"])["meas"] / r["seq"] - 1 for r in rows],
              "Semi-SP": [r["semi_sp"]["meas"] / r["seq"] - 1 for r in rows if "semi_sp" in r]}
    summ = {"config": a.config, "S": S, "g": g, "N": N, "squads": len(rows), "candidates": len(keys),
            "reps": a.reps, "split_pct": a.split_pct,
            "eq2_nsp_mape_pct": mape(eq2), "eq2_bias_pct": bias(eq2),
            "eq1_sp_mape_pct_all_splits": mape(eq1), "eq1_bias_pct_all_splits": bias(eq1),
            "eq1_sp_mape_pct_at_eq1_optimum": mape(eq1_best),
            "config_match_exact_pct": 100 * float(np.mean([r["match_exact"] for r in rows])),
            "config_match_within_2pct_pct": 100 * float(np.mean([r["match_2pct"] for r in rows])),
            "duration_vs_seq_pct": {k: (100 * float(np.mean(v)) if v else None) for k, v in vs_seq.items()},
            "kernel_slowdown_nsp": {"median": float(np.median(slow_nsp)), "p90": float(np.percentile(slow_nsp, 90)),
                                    "max": float(np.max(slow_nsp))},
            "kernel_slowdown_sp": {"median": float(np.median(slow_sp)), "p90": float(np.percentile(slow_sp, 90)),
                                   "max": float(np.max(slow_sp))},
            "paper": {"eq1_err_pct": 6.7, "eq2_err_pct": 7.1, "match_pct": 96.2,
                      "vs_seq_pct": {"NSP": -6.5, "SP": -12.9, "Semi-SP": -17.6}, "kernel_slowdown_max": 2.0}}
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump({"summary": summ, "squads": rows}, open(a.out, "w"), indent=1)
    print(json.dumps(summ, indent=1))
    ctx.close()
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
