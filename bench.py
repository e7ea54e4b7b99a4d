#!/usr/bin/env python
"""BLESS hot-path benchmark (BASELINE.json metric: avg/p99 request latency per
tenant at fixed quotas vs time-slice / static-split, and quota attainment %).

A "step" is one pass of the whole hot path over one synthetic trace: the
native dispatcher (bl_dispatch) hands each request to its GPU's context at its
arrival time, the C++ scheduler forms kernel squads from the tenants' active
requests and the SM-gated sm_100a kernels execute them (all of SURVEY.md
§8(a)).  Workload at N=1: config C2 (VGG11 quota 1/3 + ResNet50 quota 2/3,
bf16, batch 1, 224x224; BASELINE.json configs[1], the paper's Fig. 1 setup).
`value` = mean request latency (ms) under BLESS over the K timed steps; the
in-run baselines (ISO, STATIC, TEMPORAL T-cap and T-wc, UNBOUND) replay the
same traces on the same executor.  C3 and C4 are reported beside it
(`other_configs`, a load sweep each).

Multi-GPU (replicas only, no NCCL): under torchrun every rank
owns one GPU's context and dispatches its slice of one box-wide trace; without
torchrun, `--gpus N` runs one process with N contexts and one dispatcher
thread.  The ranks meet only on the host (gloo) for the barrier, the max of
the step time and the whole-job sums.

--impl reference times the oracle (oracle/: fp64 layer reference + the
discrete-event model of the policy) on the host cores instead.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synth import profile as synprof  # noqa: E402
from synth import trace as syntrace  # noqa: E402

METRIC = "avg/p99 request latency per tenant at fixed quotas vs time-slice/static-split; quota attainment %"
CONFIG_NAMES = {"C1": "tiny MLP (1/3) + tiny CNN (2/3), fp32",
                "C2": "VGG11 (1/3) + ResNet50 (2/3), bf16 batch 1",
                "C3": "ResNet50 (0.4) + VGG16 (0.3) + BERT-base s128 (0.2) + MobileNetV2 (0.1), bf16 batch 1",
                "C4": "BERT-large s384 (1/2) + ResNet152 (1/4) + DenseNet121 (1/4), bf16 batch 1, bursty",
                "C5": "per-GPU mix of C2/C3/C4 (GPU g hosts C[2 + g mod 3])"}
SQUAD_MAX = {"C1": 4, "C2": 40, "C3": 50, "C4": 10}   # C3: the paper's testbed value (L408); B200 A/B in profiles/round2/smax_defaults

# tenant (name, quota) per config -- data only, so the reference arm imports
# nothing from the product package
REF_CONFIGS = {
    "C1": [("mlp", 1 / 3), ("cnn", 2 / 3)],
    "C2": [("vgg11", 1 / 3), ("resnet50", 2 / 3)],
    "C3": [("resnet50", 0.4), ("vgg16", 0.3), ("bert_base", 0.2), ("mobilenet_v2", 0.1)],
    "C4": [("bert_large", 0.5), ("resnet152", 0.25), ("densenet121", 0.25)],
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="native", choices=["native", "reference"])
    ap.add_argument("--config", default="C2", choices=["C1", "C2", "C3", "C4", "C5"])
    ap.add_argument("--rho", type=float, default=0.5, help="per-tenant load relative to its ISO latency")
    ap.add_argument("--rhos", default="", help="comma list: per-tenant rho (PAPER.md L298 workload E, biased load)")
    ap.add_argument("--quotas", default="", help="comma list: per-tenant quota override (PAPER.md Table 2 quota sets)")
    ap.add_argument("--requests", type=int, default=100, help="requests per tenant per step (20 steps -> 2000)")
    # B200 operating point chosen by the c% x S_max sweep, the
    # way the paper picks its own empirically (§6.7).
    ap.add_argument("--squad-max", type=int, default=None,
                    help="S_max (L406-L408); default per config from the B200 sweeps: C1 4, C2 40, C3 50, C4 10")
    ap.add_argument("--split-pct", type=int, default=25)
    ap.add_argument("--squad-max-solo", type=int, default=0,
                    help="reading R36: cap of a squad with a single active request (0 = S_max)")
    ap.add_argument("--seed-all", type=int, default=1, help="reading R6: seed every active request first (1) or pick by lag only (0)")
    ap.add_argument("--ablate", type=int, default=0,
                    help="PAPER.md §6.8 ablation (R32): 1 = no multi-task scheduler, 2 = no determiner, 3 = both")
    ap.add_argument("--barrier", type=int, default=0,
                    help="squad barrier bits: 0 = every participant waits for the previous squad (L276); "
                         "1 = SM-range barrier (reading R37); 2 = arrivals join in-flight solo NSP squads (R38)")
    ap.add_argument("--lookahead-us", type=float, default=20.0)
    ap.add_argument("--dump-squads", type=int, default=0,
                    help="write the first N squads of the timed steps (picks, ranges, predicted vs measured) to out-dir")
    ap.add_argument("--max-inflight", type=int, default=2)
    ap.add_argument("--profile-reps", type=int, default=5)
    ap.add_argument("--no-baselines", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-slo", action="store_true", help="skip the SLO-mode experiment (§6.5)")
    ap.add_argument("--also", default="C2,C3,C4", help="other configs reported beside the headline (N=1 only)")
    ap.add_argument("--also-rhos", default="0.3,0.5")
    ap.add_argument("--also-requests", type=int, default=80)
    ap.add_argument("--load-profile", default="", help="reuse a saved profile table instead of profiling")
    ap.add_argument("--light", action="store_true", help="timed steps only (for ncu launch lists)")
    ap.add_argument("--out-dir", default=os.path.join(ROOT, "gpurun_out"))
    a = ap.parse_args()
    return a


# ---------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    def __init__(self, gpus):
        self.gpus, self.proc, self.lines = list(gpus), None, []

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", ",".join(str(g) for g in self.gpus),
                                          f"--query-gpu={q}", "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], 0, set()
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                mx = max(mx, float(f[1]))
            except ValueError:
                continue
            for name, v in zip(["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"], f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(name)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------------------- helpers
def squad_timeline(decisions, launches, m_of=None, S=148, barrier=0):
    """Map each BLESS decision to its launches (logged in pick order) and
    measure: squad makespan vs the predicted t_hat (Eq. 1 for SP, Eq. 2 for
    NSP; PAPER.md L214/L227 report 6.7%/7.1% error on A100) and the GPU idle
    gap between consecutive squads (L432: 20 us squad switch on A100).  Gaps
    are signed: a negative gap would be an overlap of squad s+1 with squad s
    (a broken barrier); tests/test_gpu_concurrent.py asserts there is none
    across tenants."""
    i = 0
    spans = []
    viol = 0
    prev = None
    # squad shape (a squad closes at S_max picks or on a
    # request's last kernel) and SM-time busy fraction inside squads
    npk, npt, by_last, sm_busy, sm_span = [], [], 0, 0.0, 0.0
    last = {}   # barrier bit 0: tenant -> (end of its latest chain, SM mask of that chain)
    prev_solo = False
    for d in decisions:
        ls = launches[i:i + d.n_picks]
        i += d.n_picks
        npk.append(d.n_picks)
        npt.append(d.n_part)
        if m_of is not None and d.n_picks and d.pick_kernel[d.n_picks - 1] == m_of[d.pick_tenant[d.n_picks - 1]] - 1:
            by_last += 1
        if len(ls) != d.n_picks or any(r.end_ns <= 0 or r.nsm <= 0 for r in ls):
            prev = None
            last = {}
            continue
        spans.append((min(r.start_ns for r in ls), max(r.end_ns for r in ls), d.t_hat, bool(d.config_sp)))
        sm_busy += sum((r.end_ns - r.start_ns) * r.nsm for r in ls)
        sm_span += (spans[-1][1] - spans[-1][0]) * S
        # R38 (barrier bit 2): a squad that follows a solo NSP squad may have
        # been decided at an arrival and started beside it -- not checked
        exempt = bool(barrier & 2) and prev_solo
        prev_solo = d.n_part == 1 and not d.config_sp
        if barrier & 1:
            # SM-range barrier (R37): no launch starts before the end of another
            # tenant's latest chain whose kernels used any SM this tenant's
            # chain in this squad uses
            umask = {}
            for r in ls:
                umask[r.tenant] = umask.get(r.tenant, 0) | (((1 << (r.hi - r.lo)) - 1) << r.lo)
            for r in ls:
                for t, (e, msk) in last.items():
                    if t != r.tenant and msk & umask[r.tenant] and not exempt:
                        viol += int(r.start_ns < e - 64)
            for t, msk in umask.items():
                last[t] = (max(r.end_ns for r in ls if r.tenant == t), msk)
        elif prev is not None and not exempt:   # barrier: no launch starts before ANOTHER tenant's squad-s end
            for r in ls:
                others = [e for t, e in prev.items() if t != r.tenant]
                viol += int(bool(others) and r.start_ns < max(others) - 64)
        prev = {}
        for r in ls:
            prev[r.tenant] = max(prev.get(r.tenant, 0), r.end_ns)
    if not spans:
        return {}
    err = {True: [], False: []}
    sgn = {True: [], False: []}
    gaps = [b[0] - a[1] for a, b in zip(spans, spans[1:])]
    for s, e, th, sp in spans:
        err[sp].append(abs((e - s) - th) / max(1, e - s))
        sgn[sp].append(((e - s) - th) / max(1, e - s))
    med = lambda x: float(np.median(x)) / 1e3 if x else None  # noqa: E731
    return {"squads": len(spans),
            "pred_err_sp_pct": 100 * float(np.mean(err[True])) if err[True] else None,
            "pred_err_nsp_pct": 100 * float(np.mean(err[False])) if err[False] else None,
            "pred_bias_sp_pct": 100 * float(np.mean(sgn[True])) if sgn[True] else None,
            "pred_bias_nsp_pct": 100 * float(np.mean(sgn[False])) if sgn[False] else None,
            "gap_us_median": med(gaps), "gap_us_mean": float(np.mean(gaps)) / 1e3 if gaps else None,
            "gap_us_min_signed": float(min(gaps)) / 1e3 if gaps else None,
            # squad s+1 starting before squad s ends on the SAME tenant stream is
            # the programmatic-dependent-launch prologue overlap (the kernel
            # waits in griddepcontrol.wait before touching data); a start before
            # ANOTHER tenant's end would be a broken barrier
            "pdl_overlapped_switches": int(sum(1 for g in gaps if g < 0)),
            "barrier_violations": viol,
            "makespan_us_median": med([e - s for s, e, _, _ in spans]),
            "picks_per_squad_mean": float(np.mean(npk)), "participants_per_squad_mean": float(np.mean(npt)),
            "closed_by_last_kernel_pct": 100.0 * by_last / max(1, len(decisions)) if m_of is not None else None,
            # sum over launches of (end - start) x SMs that ran a tile, over
            # sum over squads of makespan x S: the fraction of SM-time inside
            # squads that holds a running kernel (1 - bubbles)
            "in_squad_sm_busy_frac": sm_busy / sm_span if sm_span else None}


def make_trace(T_iso, rho, n, seed, bursty=False):
    """Poisson (C1-C3, C5) or bursty MMPP-2 (C4: ON 20% at 4x, OFF at 0.25x the
    mean rate, exponential dwell 20 / 80 ms) per tenant.
    ``rho`` is one load for every tenant or a per-tenant list."""
    rhos = list(rho) if isinstance(rho, (list, tuple)) else [rho] * len(T_iso)
    gaps = [T / r for T, r in zip(T_iso, rhos)]
    if bursty:
        return syntrace.mmpp2(gaps, n, seed)
    return syntrace.poisson(gaps, n, seed)


# ---------------------------------------------------------------------------- replicas
class Replica:
    """One GPU's sharing domain: ctx, tenant models, profile (L171)."""

    def __init__(self, gpu, device, cfg, args, capi, models):
        import torch
        self.gpu, self.device, self.cfg = gpu, device, cfg
        self.dtype = "fp32" if cfg == "C1" else "bf16"
        self.squad_max = args.squad_max or SQUAD_MAX.get(cfg, 20)
        with torch.cuda.device(device):
            self.ctx = capi.Ctx(device, capi.default_params(squad_max=self.squad_max))
            quotas = [float(x) for x in args.quotas.split(",")] if args.quotas and cfg == args.config else None
            self.tms = models.build_config(self.ctx, cfg, self.dtype, quotas, device=device)
        self.names = [m.name for m in self.tms]
        self.info = self.ctx.device_info()
        self.S = self.info.sm_count

    def profile(self, args, out_dir, tag):
        t0 = time.perf_counter()
        if args.load_profile and self.cfg == args.config:
            self.ctx.load_profile(args.load_profile)
        else:
            for m in self.tms:
                self.ctx.profile_tenant(m.tenant, reps=args.profile_reps)
        self.profile_s = time.perf_counter() - t0
        self.prof_path = os.path.join(out_dir, f"profile_{self.cfg}_{tag}.txt")
        self.ctx.save_profile(self.prof_path)
        self.T_iso = [self.ctx.tenant_info(m.tenant)[2] for m in self.tms]
        self.quota_sms = [self.ctx.tenant_info(m.tenant)[0] for m in self.tms]

    def params(self, capi, args, pol="BLESS", extra=None):
        return capi.default_params(squad_max=self.squad_max, policy=pol, split_pct=args.split_pct, seed_all=args.seed_all,
                                   ablate=args.ablate, squad_max_solo=args.squad_max_solo,
                                   lookahead_ns=int(args.lookahead_us * 1000),
                                   max_inflight_squads=args.max_inflight, barrier=args.barrier,
                                   **(extra or {}))


def run_box(reps, capi, params_of, box, gpu_to_ctx, tenants_filter=None):
    """Replay a box trace through the replicas this process owns, on the wall
    clock: start every ctx, dispatch each request to its GPU's ctx at its
    arrival time (native dispatcher thread, bl_dispatch), drain, stop.
    Returns per replica: per-tenant latency lists (ns), launches, decisions."""
    ctxs = [r.ctx for r in reps]
    for r in reps:
        r.ctx.reset(params_of(r))
        r.ctx.start()
    ents = [e for e in syntrace_entries(box, gpu_to_ctx)
            if tenants_filter is None or e[1] in tenants_filter]
    base = capi.now_ns() + 3_000_000
    ids = capi.dispatch(ctxs, ents, base)
    for r in reps:
        r.ctx.drain(int(300e9))
        r.ctx.stop()
    out = []
    for i, r in enumerate(reps):
        lat = {}
        for (ci, t, _), q in zip(ents, ids):
            if ci != i:
                continue
            st, info = r.ctx.poll(q)
            assert st == capi.BL_OK
            lat.setdefault(t, []).append(info.finish_ns - info.arrival_ns)
        out.append((lat, r.ctx.launches(), r.ctx.decisions()))
    return out


def syntrace_entries(box, gpu_to_ctx):
    return [(gpu_to_ctx[a.gpu], a.tenant, a.arrival_ns) for a in box if a.gpu in gpu_to_ctx]


# ---------------------------------------------------------------------------- cpu baseline (oracle)
def oracle_timing(cfg_models, decisions, prof, params, req_seen, squads_seen):
    """Time the oracle as it stands: one fp64 forward per tenant (all host
    cores, numpy BLAS) plus decide_ref on a sample of decision records (1
    core); per request = forward + decide_ref x the squads that request took
    part in (from the decision log, per tenant)."""
    from threadpoolctl import threadpool_info

    from oracle import models_ref
    from oracle.sched_ref import Active, decide_ref
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi as _c

    fwd = {}
    for i, name in enumerate(cfg_models):
        t0 = time.perf_counter()
        models_ref.FORWARD[name](1000 + i)
        fwd[name] = time.perf_counter() - t0
    dec_t = []
    for rec in decisions[:40]:
        got = _c.decision_to_tuple(rec)
        t0 = time.perf_counter()
        decide_ref(got["now"], [Active(*a) for a in got["active"]], prof, params)
        dec_t.append(time.perf_counter() - t0)
    mean_dec = float(np.mean(dec_t)) if dec_t else 0.0
    per_req = [fwd[n] + mean_dec * squads_seen[j] / max(1, req_seen[j]) for j, n in enumerate(cfg_models)]
    val = float(np.average(per_req, weights=[max(1, x) for x in req_seen])) * 1e3
    cores = max([x.get("num_threads", 1) for x in threadpool_info()] or [1])
    return {"value": val, "unit": "ms", "cores": int(cores), "kind": "oracle",
            "sample": f"1 fp64 forward per tenant ({', '.join(f'{k} {v:.2f}s' for k, v in fwd.items())}) + "
                      f"decide_ref on {len(dec_t)} logged decisions ({mean_dec * 1e6:.0f} us each, 1 core) x "
                      "the squads each tenant's request joined",
            "decide_ref_us_per_decision": mean_dec * 1e6}


def replay_all(decisions, prof_path, params):
    """Every logged decision through the oracle's decide_ref (bit-exact)."""
    from oracle.sched_ref import Active, Prof, decide_ref
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi as _c
    prof = Prof(synprof.load(prof_path))
    ok = 0
    for rec in decisions:
        got = _c.decision_to_tuple(rec)
        ref = decide_ref(got["now"], [Active(*a) for a in got["active"]], prof, params)
        ok += int(got["picks"] == [tuple(p) for p in ref.picks] and got["config"] == ref.config
                  and got["t_hat"] == ref.t_hat)
    return f"{ok}/{len(decisions)}"


# ---------------------------------------------------------------------------- roofline
def roofline_of(rep, launches_all, peaks, args):
    """Roofline of the dominant kernel (largest share of the step's device
    time).  "Kernel" = one kernel function (family, e.g. the tcgen05 conv):
    achieved = its algorithmic work / its CUDA-event launch time, each layer of
    the family timed on its tenant stream over all S SMs (bl_profile_kernel,
    back to back with PDL as inside a request), weighted by its launch count in
    the timed steps.  Also per tenant the SM-share roofline fraction (SURVEY
    §8(d)): sum_k t_roof(k, s) / sum_k t_meas(k) over the BLESS launches, with
    t_roof = max(F / (P_tc * s/S), B / (BW * s/S))."""
    ctx, S, names = rep.ctx, rep.S, rep.names
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    tc_peak = float(peaks.get("bf16_tflops", 1590.0))
    ridge = tc_peak * 1e12 / (hbm_peak * 1e9)
    peak_src = "MEASURED_PEAKS.json (burst)" if peaks else "fallback (B200_PROFILING.md)"
    busy, nlaunch = {}, {}
    for r in launches_all:
        if r.end_ns > r.start_ns and r.nsm > 0:
            busy[(r.tenant, r.kernel)] = busy.get((r.tenant, r.kernel), 0) + (r.end_ns - r.start_ns)
            nlaunch[(r.tenant, r.kernel)] = nlaunch.get((r.tenant, r.kernel), 0) + 1
    total_busy = sum(busy.values())
    fam_of = {tk: ctx.kernel_info(*tk).family.decode().split("_bf16")[0].split("_f32")[0] for tk in busy}
    fam_busy = {}
    for tk, v in busy.items():
        fam_busy[fam_of[tk]] = fam_busy.get(fam_of[tk], 0) + v
    fam = max(fam_busy, key=fam_busy.get)
    F = B = T = TR = 0.0
    per_layer = []
    for tk in busy:
        if fam_of[tk] != fam:
            continue
        ki = ctx.kernel_info(*tk)
        ev, _ = ctx.profile_kernel(tk[0], tk[1], S, reps=10)   # CUDA events on the tenant's stream
        n = nlaunch[tk]
        F += n * ki.flops
        B += n * ki.bytes
        T += n * ev
        tr = max(ki.flops / (tc_peak * 1e3), ki.bytes / hbm_peak)   # ns at the roofline
        TR += n * tr
        per_layer.append((n * ev, f"{names[tk[0]]}[{tk[1]}]", ev, tr / ev))
    if F / max(B, 1.0) >= ridge:
        bound, unit, achieved, peak = "tensor", "TFLOP/s", F / T / 1e3, tc_peak
    else:
        bound, unit, achieved, peak = "hbm", "GB/s", B / T, hbm_peak
    per_layer.sort(reverse=True)
    nl = sum(nlaunch[tk] for tk in busy if fam_of[tk] == fam)
    traffic = None
    tpath = os.path.join(ROOT, "profiles", f"traffic_{rep.cfg}.json")
    if os.path.exists(tpath):
        tl = json.load(open(tpath))["layers"]
        keys = [(tk, f"{names[tk[0]]}[{tk[1]}]") for tk in busy if fam_of[tk] == fam]
        if all(k in tl and tl[k]["dram_read"] is not None for _, k in keys):
            traffic = sum(nlaunch[tk] * (tl[k]["dram_read"] + tl[k]["dram_write"]) for tk, k in keys) / max(1, nl)
    roof = {"bound": bound, "achieved": achieved, "peak": peak, "unit": unit, "frac": achieved / peak,
            "traffic": traffic, "traffic_source": f"profiles/traffic_{rep.cfg}.json" if traffic else None,
            "kernel": fam, "layers": len(per_layer),
            "algorithmic_flops_per_launch": F / max(1, nl), "algorithmic_bytes_per_launch": B / max(1, nl),
            "event_avg_ns_per_launch": T / max(1, nl), "roofline_time_frac": TR / T,
            "instep_share": fam_busy[fam] / max(total_busy, 1),
            "top_layers": [{"layer": nm, "event_ns": round(ev), "roofline_time_frac": round(fr, 3)}
                           for _, nm, ev, fr in per_layer[:5]],
            "peak_source": peak_src}
    # the same family at the SM range its launches actually got in the timed
    # BLESS steps (median hi - lo per layer), against the SM-share peak
    # P * s/S ("against the chip's peak scaled by the tenant's
    # SM share")
    rng = {}
    for r in launches_all:
        if r.end_ns > r.start_ns and r.nsm > 0 and fam_of.get((r.tenant, r.kernel)) == fam:
            rng.setdefault((r.tenant, r.kernel), []).append(r.hi - r.lo)
    Fr = Tr = Pr = 0.0
    tensor = bound == "tensor"
    for tk, sizes in rng.items():
        s_med = int(np.median(sizes))
        ki = ctx.kernel_info(*tk)
        ev, _ = ctx.profile_kernel(tk[0], tk[1], s_med, reps=10)
        n = nlaunch[tk]
        Fr += n * (ki.flops if tensor else ki.bytes)
        Tr += n * ev
        Pr += n * ev * ((tc_peak if tensor else hbm_peak) * s_med / S)   # time-weighted share of the peak
    if Tr > 0:
        peak_share = Pr / Tr
        ach = Fr / Tr / 1e3 if tensor else Fr / Tr
        roof["at_range"] = {"achieved": ach, "peak_share": peak_share, "unit": unit,
                            "frac": ach / peak_share,
                            "note": "each layer timed on its median SM range in the timed steps; peak = "
                                    f"measured {'bf16' if tensor else 'HBM'} peak x s/S, time-weighted"
                                    + ("" if tensor else " (HBM is not partitioned by SMs: a share can "
                                                         "exceed 1, SURVEY §8(d))")}
    hb = [tk for tk in busy if (lambda k: k.flops / max(k.bytes, 1.0) < ridge)(ctx.kernel_info(*tk))]
    if hb:
        tk = max(hb, key=lambda x: busy[x] / nlaunch[x])
        ki = ctx.kernel_info(*tk)
        ev, _ = ctx.profile_kernel(tk[0], tk[1], S, reps=20)
        roof["hbm_kernel"] = {"kernel": f"{names[tk[0]]}[{tk[1]}] {ki.family.decode()}", "bound": "hbm",
                              "achieved": ki.bytes / ev, "peak": hbm_peak, "unit": "GB/s",
                              "frac": ki.bytes / ev / hbm_peak, "algorithmic_bytes": ki.bytes, "event_ns": ev}
        if os.path.exists(tpath):
            rec = json.load(open(tpath))["layers"].get(f"{names[tk[0]]}[{tk[1]}]")
            if rec and rec["dram_read"] is not None:
                roof["hbm_kernel"]["traffic"] = rec["dram_read"] + rec["dram_write"]
    kinfo = {(m.tenant, k): ctx.kernel_info(m.tenant, k) for m in rep.tms for k in range(len(m.layers))}
    share = {}
    for r in launches_all:
        if r.end_ns <= r.start_ns or r.nsm <= 0:
            continue
        ki2 = kinfo[(r.tenant, r.kernel)]
        s_used = max(1, r.hi - r.lo)
        t_roof = max(ki2.flops / (tc_peak * 1e12 * s_used / S), ki2.bytes / (hbm_peak * 1e9 * s_used / S)) * 1e9
        a = share.setdefault(names[r.tenant], [0.0, 0.0])
        a[0] += t_roof
        a[1] += r.end_ns - r.start_ns
    return roof, {nm: tr_ / tm_ for nm, (tr_, tm_) in share.items()}


# ---------------------------------------------------------------------------- other configs (N=1)
def other_config(cfg, args, capi, models, metrics, out_dir, rhos=None):
    """A compact run of another config beside the headline: profile, then per
    load rho BLESS / STATIC / TEMPORAL T-wc / ISO on seeds 1-3 (same traces):
    mean latency per policy, attainment per tenant, deviation (L320).  For the
    headline config itself: the loads other than the headline's (its load
    boundary)."""
    rep = Replica(0, 0, cfg, args, capi, models)
    rep.squad_max = args.squad_max or SQUAD_MAX[cfg]
    rep.profile(argparse.Namespace(**{**vars(args), "load_profile": ""}), out_dir, "also")
    res = {"workload": f"{cfg}: {CONFIG_NAMES[cfg]}", "squad_max": rep.squad_max, "T_iso_profile_ms":
           {n: t / 1e6 for n, t in zip(rep.names, rep.T_iso)}, "rho": {}}
    nt = len(rep.tms)
    for rho in (rhos if rhos is not None else [float(x) for x in args.also_rhos.split(",") if x]):
        lat = {}
        for pol, extra in (("BLESS", None), ("STATIC", None), ("TEMPORAL_Twc", {"temporal_work_conserving": 1}),
                           ("ISO", None)):
            acc = {j: [] for j in range(nt)}
            for seed in (1, 2, 3):
                tr = make_trace(rep.T_iso, rho, args.also_requests, seed, cfg == "C4")
                box = [syntrace.BoxArrival(a.arrival_ns, 0, a.tenant) for a in tr]
                name = pol.split("_")[0]
                if pol == "ISO":
                    for j in range(nt):
                        (l, _, _), = run_box([rep], capi, lambda r: r.params(capi, args, "ISO"), box, {0: 0}, {j})
                        acc[j].extend(l.get(j, []))
                else:
                    (l, _, _), = run_box([rep], capi, lambda r: r.params(capi, args, name, extra), box, {0: 0})
                    for j, v in l.items():
                        acc[j].extend(v)
            lat[pol] = acc
        means = {p: {j: float(np.mean(v)) for j, v in acc.items()} for p, acc in lat.items()}
        allm = {p: float(np.mean([x for v in acc.values() for x in v])) / 1e6 for p, acc in lat.items()}
        att = {rep.names[j]: metrics.attainment_pct(means["ISO"][j], means["BLESS"][j]) for j in range(nt)}
        res["rho"][str(rho)] = {
            "mean_ms": allm,
            "attainment_pct": att, "min_attainment_pct": min(att.values()),
            "deviation_ms": {p: metrics.latency_deviation(means[p], means["ISO"]) / 1e6 for p in means if p != "ISO"},
            "bless_beats_static": allm["BLESS"] < allm["STATIC"], "bless_beats_twc": allm["BLESS"] < allm["TEMPORAL_Twc"],
            "time_domain_demand_D": float(rho * sum(_full_over_quota(rep)))}
    rep.ctx.close()
    return res


def _full_over_quota(rep):
    """T_j(S) / T_j(quota SMs) from the profile: the time-domain demand factor
    per tenant (D = sum_j rho_j T_j(S)/T_j(q_j))."""
    out = []
    for m, Tq in zip(rep.tms, rep.T_iso):
        TS = sum(rep.ctx.get_profile_row(m.tenant, k, rep.S)[0][rep.S - 1] for k in range(len(m.layers)))
        out.append(TS / max(1, Tq))
    return out


# ---------------------------------------------------------------------------- native arm
def native(args):
    import torch

    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build as bld
    bld.build(verbose=False)
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi, metrics, models, replicas

    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    dist = None
    # BLESS_BENCH_DEVICE=d puts every replica on device d: a plumbing check of
    # the multi-rank path on a one-GPU box (replicas never wait on each other;
    # its numbers are not scaling measurements)
    force_dev = os.environ.get("BLESS_BENCH_DEVICE")
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo")   # host-side barrier and reductions only (no NCCL: nothing shards)
        gpus = [(rank, local if force_dev is None else int(force_dev))]
    else:
        gpus = [(g, g if force_dev is None else int(force_dev)) for g in range(max(1, args.gpus))]
    n_box = world if world > 1 else len(gpus)
    os.makedirs(args.out_dir, exist_ok=True)
    # tcgen05 tile configurations are autotuned at registration; a saved profile
    # is only valid with the configurations it was measured with (tctune file)
    if args.load_profile:
        tune = args.load_profile.replace("profile_", "tctune_")
        if not os.path.exists(tune):
            raise SystemExit(f"--load-profile needs its tuning file {tune}")
    else:
        tune = os.path.join(args.out_dir, f"tctune_{args.config}_gpu{rank}.txt")   # pairs with profile_*_gpu{g}
        if os.path.exists(tune):
            os.remove(tune)
    os.environ["BLESS_TC_TUNE_FILE"] = tune

    reps = []
    for g, dev in gpus:
        torch.cuda.set_device(dev)
        reps.append(Replica(g, dev, replicas.plan(g, args.config).config, args, capi, models))
    for r in reps:
        r.profile(args, args.out_dir, f"gpu{r.gpu}")
    gpu_to_ctx = {r.gpu: i for i, r in enumerate(reps)}
    # box-wide per-GPU T_iso -> the same box trace on every rank
    tiso = {}
    for part in replicas.gather({r.gpu: (r.T_iso, r.cfg) for r in reps}, dist):
        tiso.update(part)
    rho_t = [float(x) for x in args.rhos.split(",")] if args.rhos else None

    def box_of(seed):
        gaps, bursty = [], []
        for g in range(n_box):
            T, cfg = tiso[g]
            rr = rho_t if (rho_t and cfg == args.config) else [args.rho] * len(T)
            gaps.append([t / x for t, x in zip(T, rr)])
            bursty.append(cfg == "C4")
        return syntrace.box_trace(gaps, args.requests, seed, bursty)

    def step(seed, pol="BLESS", filt=None, extra=None):
        return run_box(reps, capi, lambda r: r.params(capi, args, pol, extra), box_of(seed), gpu_to_ctx, filt)

    flush = [torch.empty(256 << 20, dtype=torch.uint8, device=f"cuda:{r.device}") for r in reps]

    def flush_l2():
        for f in flush:
            f.zero_()

    for w in range(args.warmup):
        flush_l2()
        step(100 + w)

    # ---------------- timed region: K BLESS steps
    nrep = len(reps)
    lat_all = [{j: [] for j in range(len(r.tms))} for r in reps]
    seed_lat = {}
    launches_all = [[] for _ in reps]
    decisions_all = [[] for _ in reps]
    timelines = []
    replicas.barrier(dist)
    for r in reps:
        torch.cuda.synchronize(r.device)
    with ClockSampler([r.device for r in reps]) as clk:
        t0 = time.perf_counter()
        for k in range(args.steps):
            flush_l2()
            sd = 1 + k % 3
            out = step(sd)
            for i, (lat, launches, decisions) in enumerate(out):
                for j, v in lat.items():
                    lat_all[i][j].extend(v)
                    seed_lat.setdefault(sd, []).extend(v)
                launches_all[i].extend(launches)
                decisions_all[i].extend(decisions)
                if i == 0:
                    timelines.append((decisions, launches))
        for r in reps:
            torch.cuda.synchronize(r.device)
        t1 = time.perf_counter()
    step_ms = replicas.max_over_ranks((t1 - t0) * 1e3 / args.steps, dist)
    replicas.barrier(dist)
    n_local = sum(len(v) for la in lat_all for v in la.values())
    agg = replicas.sum_over_ranks({"n": n_local, "lat_sum": float(sum(x for la in lat_all for v in la.values()
                                                                     for x in v))}, dist)
    n_req = int(agg["n"])
    mean_ms = agg["lat_sum"] / max(1.0, agg["n"]) / 1e6
    gpu_launches = int(replicas.sum_over_ranks({"l": sum(len(x) for x in launches_all)}, dist)["l"])
    if args.light:
        if rank == 0:
            print(json.dumps({"metric": METRIC, "value": mean_ms, "unit": "ms", "light": True,
                              "gpu_launches": gpu_launches, "ms_per_step": step_ms}))
        for r in reps:
            r.ctx.close()
        return

    # ---------------- in-run baselines on the SAME traces as the timed steps
    # (each distinct seed once, weighted by how often the timed steps used it)
    seeds = [1 + k % 3 for k in range(args.steps)]
    mult = {sd: seeds.count(sd) for sd in sorted(set(seeds))}

    def run_seeds(pol, filt_of=None, extra=None):
        out = [{} for _ in reps]
        for sd, n in mult.items():
            if filt_of is None:
                res = step(sd, pol, None, extra)
                for i, (l, _, _) in enumerate(res):
                    for j, v in l.items():
                        out[i].setdefault(j, []).extend(v * n)
            else:
                for filt in filt_of:
                    res = step(sd, pol, filt, extra)
                    for i, (l, _, _) in enumerate(res):
                        for j, v in l.items():
                            out[i].setdefault(j, []).extend(v * n)
        return out

    def key(i, j):
        return reps[i].names[j] if nrep == 1 else f"gpu{reps[i].gpu}:{reps[i].names[j]}"

    per_tenant, base, iso_means, base_lat, deviation = {}, {}, {}, {}, {}
    bless_means = {(i, j): float(np.mean(v)) for i in range(nrep) for j, v in lat_all[i].items() if v}
    if not args.no_baselines:
        maxt = max(len(r.tms) for r in reps)
        iso = run_seeds("ISO", [{j} for j in range(maxt)])
        iso_means = {(i, j): float(np.mean(v)) for i in range(nrep) for j, v in iso[i].items()}
        base["ISO"] = {key(i, j): metrics.summary_ms(v) for i in range(nrep) for j, v in iso[i].items()}
        base["ISO"]["all_mean_ms"] = float(np.mean([x for d in iso for v in d.values() for x in v])) / 1e6
        runs = {"STATIC": ("STATIC", {}), "TEMPORAL_Tcap": ("TEMPORAL", {}),
                "TEMPORAL_Twc": ("TEMPORAL", {"temporal_work_conserving": 1}), "UNBOUND": ("UNBOUND", {})}
        for label, (pol, extra) in runs.items():
            lsb = run_seeds(pol, None, extra)
            base_lat[label] = lsb
            base[label] = {key(i, j): metrics.summary_ms(v) for i in range(nrep) for j, v in lsb[i].items()}
            base[label]["all_mean_ms"] = float(np.mean([x for d in lsb for v in d.values() for x in v])) / 1e6
            means = {(i, j): float(np.mean(v)) for i in range(nrep) for j, v in lsb[i].items()}
            deviation[label] = metrics.latency_deviation(means, iso_means) / 1e6
        base["seeds"] = mult
        deviation["BLESS"] = metrics.latency_deviation(bless_means, iso_means) / 1e6
    for i in range(nrep):
        for j in range(len(reps[i].tms)):
            s = metrics.summary_ms(lat_all[i][j])
            if iso_means:
                s["attainment_pct"] = metrics.attainment_pct(iso_means[(i, j)], bless_means[(i, j)])
            s["quota_sms"] = reps[i].quota_sms[j]
            s["T_iso_profile_ms"] = reps[i].T_iso[j] / 1e6
            per_tenant[key(i, j)] = s
    atts = [s["attainment_pct"] for s in per_tenant.values() if "attainment_pct" in s]

    # ---------------- SLO mode (§6.5): QoS target replaces T[n%] in
    # the progress order; violation rate = share of requests over the target
    slo = None
    if not args.no_baselines and not args.no_slo:
        slo = {}
        for label, fac in (("tight", (1.2, 2.0)), ("loose", (1.5, 3.0))):
            tgt = {(i, j): int(fac[j % 2] * iso_means[(i, j)]) for i in range(nrep) for j in range(len(reps[i].tms))}
            for i, r in enumerate(reps):
                for m in r.tms:
                    r.ctx.set_slo(m.tenant, tgt[(i, m.tenant)])
            ls = run_seeds("BLESS")
            for r in reps:
                for m in r.tms:
                    r.ctx.set_slo(m.tenant, 0)

            def viol(l):
                n = sum(len(v) for d in l for v in d.values())
                return 100.0 * sum(sum(1 for x in v if x > tgt[(i, j)]) for i, d in enumerate(l)
                                   for j, v in d.items()) / max(1, n)
            row = {"targets_ms": {key(i, j): v / 1e6 for (i, j), v in tgt.items()},
                   "factors_x_measured_ISO_mean": list(fac),
                   "violation_pct": {"BLESS_SLO": viol(ls), "BLESS": viol(lat_all)}}
            row["violation_pct"].update({k: viol(v) for k, v in base_lat.items()})
            row["BLESS_SLO_mean_ms"] = {key(i, j): float(np.mean(v)) / 1e6 for i, d in enumerate(ls)
                                        for j, v in d.items()}
            slo[label] = row

    # ---------------- e2e: same metric with host buffers (H2D input, D2H output per request)
    pinned = []
    for r in reps:
        for m in r.tms:
            hin = torch.empty(m.input.shape, dtype=m.input.dtype).pin_memory()
            hin.copy_(m.input.cpu())
            hout = torch.empty(m.output.shape, dtype=m.output.dtype).pin_memory()
            pinned += [hin, hout]
            r.ctx.set_tenant_io(m.tenant, hin.data_ptr(), m.input.data_ptr(), hin.numel() * hin.element_size(),
                                m.output.data_ptr(), hout.data_ptr(), hout.numel() * hout.element_size())
    le = step(1)
    h2d = sum(r.tms[j].input.numel() * r.tms[j].input.element_size() * len(v)
              for r, (l, _, _) in zip(reps, le) for j, v in l.items())
    d2h = sum(r.tms[j].output.numel() * r.tms[j].output.element_size() * len(v)
              for r, (l, _, _) in zip(reps, le) for j, v in l.items())
    e2e_all = [x for (l, _, _) in le for v in l.values() for x in v]
    e2e = {"value": float(np.mean(e2e_all)) / 1e6, "unit": "ms", "h2d_bytes_per_step": int(h2d),
           "d2h_bytes_per_step": int(d2h), "requests": len(e2e_all),
           "path": "bl_set_tenant_io: pinned host input -> device per request, output -> pinned host; a request "
                   "completes when its output has landed in host memory"}
    for r in reps:
        for m in r.tms:
            r.ctx.set_tenant_io(m.tenant, 0, 0, 0, 0, 0, 0)

    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    roofline, share = roofline_of(reps[0], launches_all[0], peaks, args)
    for nm, fr in share.items():
        per_tenant[nm if nrep == 1 else f"gpu{reps[0].gpu}:{nm}"]["sm_share_roofline_frac"] = fr

    # ---------------- host cost of the C++ scheduler (L436), 1 core
    dec = decisions_all[0]
    decide_cost = None
    if dec:
        r0 = reps[0]
        r0.ctx.reset(r0.params(capi, args))
        ns, picks = r0.ctx.time_decide(dec, reps=3)
        decide_cost = {"us_per_decision": ns / (3 * len(dec)) / 1e3, "us_per_kernel": ns / max(1, picks) / 1e3,
                       "decisions": len(dec), "cores": 1,
                       "paper_us_per_kernel": 6.7, "paper_host": "AMD EPYC 7302 (L282, L436)"}

    # ---------------- cpu baseline (oracle) + full decision replay, rank 0 at N=1 only
    cpu = None
    replay_ok = None
    if rank == 0:
        from oracle.sched_ref import Params, Prof
        r0 = reps[0]
        prm = Params(squad_max=r0.squad_max, split_pct=args.split_pct, ablate=args.ablate,
                     squad_max_solo=args.squad_max_solo, seed_all=bool(args.seed_all))
        replay_ok = replay_all(dec, r0.prof_path, prm)
        if world == 1 and nrep == 1 and not args.no_cpu_baseline:
            prof = Prof(synprof.load(r0.prof_path))
            sq_seen = [sum(1 for d in dec if j in [d.part_tenant[x] for x in range(d.n_part)])
                       for j in range(len(r0.tms))]
            cpu = oracle_timing(r0.names, dec, prof, prm, [len(lat_all[0][j]) for j in range(len(r0.tms))], sq_seen)

    tl = [squad_timeline(d, l, [len(m.layers) for m in reps[0].tms], reps[0].S, args.barrier) for d, l in timelines]
    if args.dump_squads and timelines and rank == 0:
        dump, (dd, ll) = [], timelines[0]
        i = 0
        for d in dd[:args.dump_squads]:
            ls = ll[i:i + d.n_picks]
            i += d.n_picks
            t0 = min(r.start_ns for r in ls) if ls else 0
            dump.append({"now": d.now, "t_hat_us": d.t_hat / 1e3, "t_nsp_us": d.t_nsp / 1e3, "sp": bool(d.config_sp),
                         "active": [(d.act_tenant[x], d.act_next[x], d.act_arrival[x]) for x in range(d.n_active)],
                         "p": [d.part_p[x] for x in range(d.n_part)] if d.config_sp else None,
                         "launches": [(r.tenant, r.kernel, r.lo, r.hi, r.nsm, round((r.start_ns - t0) / 1e3, 1),
                                       round((r.end_ns - t0) / 1e3, 1)) for r in ls]})
        with open(os.path.join(args.out_dir, f"squads_{args.config}.json"), "w") as f:
            json.dump(dump, f)
    tl = [t for t in tl if t]
    timeline = {}
    if tl:
        timeline = {k: (float(np.mean([t[k] for t in tl if t.get(k) is not None]))
                        if any(t.get(k) is not None for t in tl) else None)
                    for k in tl[0] if k not in ("squads", "pdl_overlapped_switches", "barrier_violations",
                                                "gap_us_min_signed")}
        timeline["squads"] = int(sum(t["squads"] for t in tl))
        timeline["pdl_overlapped_switches"] = int(sum(t["pdl_overlapped_switches"] for t in tl))
        timeline["barrier_violations"] = int(sum(t["barrier_violations"] for t in tl))
        mins = [t["gap_us_min_signed"] for t in tl if t.get("gap_us_min_signed") is not None]
        timeline["gap_us_min_signed"] = min(mins) if mins else None

    others = {}
    if rank == 0 and world == 1 and nrep == 1 and args.also and not args.no_baselines:
        for cfg in [c for c in args.also.split(",") if c]:
            if cfg == args.config:   # the headline config at the other loads (not when --rhos biases it)
                rl = [float(x) for x in args.also_rhos.split(",") if x and abs(float(x) - args.rho) > 1e-9]
                if rl and not args.rhos:
                    others[cfg] = other_config(cfg, args, capi, models, metrics, args.out_dir, rl)
            else:
                others[cfg] = other_config(cfg, args, capi, models, metrics, args.out_dir)

    fallbacks = sum(r.fallback for la in launches_all for r in la)
    seed_means = {str(sd): float(np.mean(v)) / 1e6 for sd, v in sorted(seed_lat.items())}
    bmean = {k: v["all_mean_ms"] for k, v in base.items() if isinstance(v, dict) and "all_mean_ms" in v}
    r0 = reps[0]
    out = {
        "metric": METRIC, "value": mean_ms, "unit": "ms", "n_gpus": n_box, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": step_ms, "higher_is_better": False, "scaling": "weak",
        "vs_baseline": None, "dtype": "bf16" if r0.dtype == "bf16" else "f32", "data": "synthetic",
        "config": {"workload": f"{args.config}: {CONFIG_NAMES[args.config]}",
                   "per_gpu_configs": {str(g): tiso[g][1] for g in sorted(tiso)},
                   "trace": f"{'MMPP-2 bursty' if args.config == 'C4' else 'Poisson'} rho={args.rhos or args.rho} "
                   f"per tenant, {args.requests} requests/tenant/step, seeds 1-3, box-wide trace routed by the "
                   "native dispatcher (bl_dispatch)", "squad_max": r0.squad_max,
                   "split_pct": args.split_pct, "ablate": args.ablate, "squad_max_solo": args.squad_max_solo, "barrier": args.barrier,
                   "seed_all": args.seed_all,
                   "parallelism": f"replicas x{n_box} (no collective; "
                                  f"{'one process per GPU, gloo host barrier' if world > 1 else 'one process'})",
                   "quotas": [m.quota for m in r0.tms],
                   "l2": "256 MiB buffer written between timed steps (> 126 MB L2); VGG11 weights 266 MB > L2"},
        "min_attainment_pct": min(atts) if atts else None,
        "vs_static": mean_ms / bmean["STATIC"] if "STATIC" in bmean else None,
        "vs_temporal_twc": mean_ms / bmean["TEMPORAL_Twc"] if "TEMPORAL_Twc" in bmean else None,
        "vs_temporal_tcap": mean_ms / bmean["TEMPORAL_Tcap"] if "TEMPORAL_Tcap" in bmean else None,
        "vs_unbound": mean_ms / bmean["UNBOUND"] if "UNBOUND" in bmean else None,
        "deviation_ms": deviation or None,
        "seed_means_ms": seed_means,
        "seed_std_ms": float(np.std(list(seed_means.values()))) if seed_means else None,
        "per_tenant": per_tenant, "baselines": base, "slo": slo,
        "requests_per_s": n_req / (step_ms * args.steps / 1e3), "requests": n_req,
        "e2e": e2e, "gpu_launches": gpu_launches, "roofline": roofline, "cpu_baseline": cpu,
        "clocks": clk.summary(),
        "scheduler": {"decisions": sum(len(d) for d in decisions_all),
                      "sp_squads": sum(1 for dd in decisions_all for d in dd if d.config_sp),
                      "fallback_launches": fallbacks, "oracle_replay_bit_exact": replay_ok,
                      "decide_cost": decide_cost, "profile_s": r0.profile_s, "timeline": timeline},
        "other_configs": others or None,
        "device": {"sm_count": r0.S, "globaltimer_res_ns": r0.info.globaltimer_res_ns, "host_cores": os.cpu_count()},
    }
    # compact summary again at the END of the line (a truncated tail keeps it)
    out["summary"] = {"value_ms": mean_ms, "min_attainment_pct": out["min_attainment_pct"],
                      "attainment_pct": {k: v.get("attainment_pct") for k, v in per_tenant.items()},
                      "mean_ms": {"BLESS": mean_ms, **bmean}, "vs_static": out["vs_static"],
                      "vs_temporal_twc": out["vs_temporal_twc"], "vs_temporal_tcap": out["vs_temporal_tcap"],
                      "vs_unbound": out["vs_unbound"], "deviation_ms": out["deviation_ms"],
                      "roofline_frac": roofline["frac"], "replay": replay_ok,
                      "other_configs": {c: {rho: {"BLESS": x["mean_ms"]["BLESS"], "STATIC": x["mean_ms"]["STATIC"],
                                                  "min_attainment_pct": x["min_attainment_pct"]}
                                            for rho, x in o["rho"].items()} for c, o in others.items()}}
    if rank == 0:
        print(json.dumps(out))
    for r in reps:
        r.ctx.close()
    if dist:
        dist.destroy_process_group()


# ---------------------------------------------------------------------------- reference arm (oracle)
def reference(args):
    rank = int(os.environ.get("RANK", 0))
    if rank != 0:
        return
    from oracle import des, models_ref
    from oracle.sched_ref import Params, Prof
    from threadpoolctl import threadpool_info

    cfg = "C2" if args.config == "C5" else args.config
    args.config = cfg
    squad_max = args.squad_max or SQUAD_MAX[cfg]
    tenants = REF_CONFIGS[cfg]
    names = [n for n, _ in tenants]
    # profile table: the last B200 profile committed under profiles/, else a synthetic stand-in
    cand = os.path.join(ROOT, "profiles", f"profile_{cfg}_b200.txt")
    if os.path.exists(cand):
        prof = Prof(synprof.load(cand))
        src = cand
    else:
        g = np.random.Generator(np.random.PCG64(7))
        tn = [synprof.random_tenant(n, int(round(q * 1e6)), 40, 148, g, 1e6, 0.6, 0.2, 1500) for n, q in tenants]
        prof = Prof(synprof.ProfileFile(148, 4, tn))
        src = "synthetic"
    vals = []
    for it in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        trace = make_trace(prof.T, args.rho, max(4, args.requests // 20), 1 + it % 3, cfg == "C4")
        des.run_bless(trace, prof, Params(squad_max=squad_max, split_pct=args.split_pct, ablate=args.ablate))
        t_dec = time.perf_counter() - t0
        fw = {}
        for i, n in enumerate(names):
            t1 = time.perf_counter()
            models_ref.FORWARD[n](1000 + i)
            fw[n] = time.perf_counter() - t1
        per_req = np.mean([fw[n] for n in names]) + t_dec / max(1, len(trace))
        if it >= args.warmup:
            vals.append(per_req * 1e3)
    v = float(np.mean(vals))
    cores = max([x.get("num_threads", 1) for x in threadpool_info()] or [1])
    out = {"impl": "reference", "metric": METRIC, "value": v, "unit": "ms", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "higher_is_better": False, "scaling": "weak",
           "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "config": {"workload": f"{args.config}: {CONFIG_NAMES[args.config]}", "profile": src},
           "cpu_baseline": {"value": v, "unit": "ms", "cores": int(cores), "kind": "oracle",
                            "sample": f"per step: DES+decide_ref over a {max(4, args.requests // 20)}-request/tenant "
                                      "trace + one fp64 forward per tenant"},
           "e2e": {"value": v, "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out))


if __name__ == "__main__":
    a = parse()
    if a.impl == "reference":
        reference(a)
    else:
        native(a)
