"""Profile-table file format and synthetic (analytic) profile tables.

File format ``profile.txt`` (whitespace separated, one record per line; read by
both the C++ runtime ``bl_load_profile`` and the Python oracle)::

    bless-profile 1
    S <S> g <g>
    tenants <n>
    tenant <name> <quota_ppm> <m>
    slo <ns>                                     (optional: SLO mode target)
    io <in_ns> <out_ns>                          (optional: per-request H2D / D2H copy time)
    tau <sms> <tau_0> ... <tau_{m-1}>            (optional: measured progress, reading R35)
    kernel <name> <d> <t_1> <t_2> ... <t_S>      (m lines per tenant)

``t_s`` is the kernel's duration in integer ns when confined to s SMs
(s = 1..S, PAPER.md L157 ``t[n%][k]`` at every SM count); ``d``
is the number of distinct SMs it used in an unrestricted run (PAPER.md L157
``d%``).  Quotas are integer parts-per-million (SURVEY.md
§8(b)).  Derived quantities (quota_sms, tau, T) are NOT stored: each side
derives them independently.

The synthetic tables below are *inputs* (the survey's analytic "Risk" model,
SURVEY.md §8(c)): ``t[k][s] = floor(W_k / min(s, d_k)) + c0``.  They do not
implement any part of the method.
"""
from __future__ import annotations

import json
from dataclasses import dataclass, field
from typing import List, Sequence

import numpy as np


@dataclass
class KernelRow:
    name: str
    d: int
    t: List[int]  # t[s-1] = duration on s SMs, s = 1..S


@dataclass
class TenantRows:
    name: str
    quota_ppm: int
    kernels: List[KernelRow] = field(default_factory=list)
    slo_ns: int = 0   # optional "slo <ns>" line (SLO mode); 0 = none
    io_in: int = 0    # optional "io <in_ns> <out_ns>" line: per-request H2D / D2H copy durations
    io_out: int = 0
    tau_sms: int = 0  # optional "tau <sms> <tau_0..tau_{m-1}>" line: time from the start of an isolated
    tau: List[int] = field(default_factory=list)   # run on tau_sms SMs to the end of kernel k (R35)


@dataclass
class ProfileFile:
    S: int
    g: int
    tenants: List[TenantRows]


def save(path: str, pf: ProfileFile) -> None:
    lines = ["bless-profile 1", f"S {pf.S} g {pf.g}", f"tenants {len(pf.tenants)}"]
    for tn in pf.tenants:
        lines.append(f"tenant {tn.name} {int(tn.quota_ppm)} {len(tn.kernels)}")
        if tn.slo_ns:
            lines.append(f"slo {int(tn.slo_ns)}")
        if tn.io_in or tn.io_out:
            lines.append(f"io {int(tn.io_in)} {int(tn.io_out)}")
        if tn.tau:
            lines.append("tau %d %s" % (int(tn.tau_sms), " ".join(str(int(v)) for v in tn.tau)))
        for k in tn.kernels:
            assert len(k.t) == pf.S, (len(k.t), pf.S)
            lines.append("kernel %s %d %s" % (k.name, int(k.d), " ".join(str(int(v)) for v in k.t)))
    with open(path, "w") as f:
        f.write("\n".join(lines) + "\n")


def load(path: str) -> ProfileFile:
    with open(path) as f:
        toks = [ln.split() for ln in f if ln.strip()]
    assert toks[0] == ["bless-profile", "1"], toks[0]
    S, g = int(toks[1][1]), int(toks[1][3])
    n = int(toks[2][1])
    i = 3
    tenants = []
    for _ in range(n):
        _, name, ppm, m = toks[i]
        i += 1
        tn = TenantRows(name, int(ppm))
        while i < len(toks) and toks[i][0] in ("slo", "io", "tau"):
            if toks[i][0] == "slo":
                tn.slo_ns = int(toks[i][1])
            elif toks[i][0] == "io":
                tn.io_in, tn.io_out = int(toks[i][1]), int(toks[i][2])
            else:
                tn.tau_sms = int(toks[i][1])
                tn.tau = [int(v) for v in toks[i][2:2 + int(m)]]
            i += 1
        for _ in range(int(m)):
            row = toks[i]
            i += 1
            assert row[0] == "kernel"
            tn.kernels.append(KernelRow(row[1], int(row[2]), [int(v) for v in row[3:3 + S]]))
        tenants.append(tn)
    return ProfileFile(S, g, tenants)


def analytic_kernel(name: str, W: int, d: int, S: int, c0: int = 0) -> KernelRow:
    """t[s] = floor(W / min(s, d)) + c0 for s = 1..S (input model, not method)."""
    return KernelRow(name, int(d), [int(W) // min(s, int(d)) + int(c0) for s in range(1, S + 1)])


def random_tenant(name: str, quota_ppm: int, m: int, S: int, rng: np.random.Generator,
                  solo_ns: float, d_mean_frac: float, d_sd_frac: float, c0: int) -> TenantRows:
    """Survey Risk-model tenant: W_k ~ Exp(1) scaled so sum_k t[k][S] ~= solo_ns,
    d_k ~ N(f*S, sd*S) clipped to [1, S]."""
    w = rng.exponential(1.0, size=m)
    d = np.clip(np.rint(rng.normal(d_mean_frac * S, d_sd_frac * S, size=m)), 1, S).astype(int)
    per_s = np.array([wk / dk for wk, dk in zip(w, d)])  # ~ t[k][S] before scaling
    scale = max(solo_ns - c0 * m, 1.0) / max(per_s.sum(), 1e-12)
    W = np.maximum(1, np.rint(w * scale)).astype(np.int64)
    return TenantRows(name, int(quota_ppm),
                      [analytic_kernel(f"{name}_k{i}", int(W[i]), int(d[i]), S, c0) for i in range(m)])


def random_table(S: int, g: int, quotas_ppm: Sequence[int], m: Sequence[int], seed: int,
                 tmax: int = 1000, noisy: bool = True) -> ProfileFile:
    """Fully random small tables for property tests (non-monotone allowed,
    SURVEY.md §7 hard part 7: "non-monotone t[k][s] is legal data")."""
    rng = np.random.Generator(np.random.PCG64(seed))
    tenants = []
    for j, (q, mj) in enumerate(zip(quotas_ppm, m)):
        tn = TenantRows(f"t{j}", int(q))
        for k in range(mj):
            d = int(rng.integers(1, S + 1))
            if noisy:
                t = [int(v) for v in rng.integers(1, tmax + 1, size=S)]
            else:
                W = int(rng.integers(1, tmax * d + 1))
                t = [W // min(s, d) + 1 for s in range(1, S + 1)]
            tn.kernels.append(KernelRow(f"t{j}k{k}", d, t))
        tenants.append(tn)
    return ProfileFile(S, g, tenants)


def save_params(path: str, params: dict) -> None:
    with open(path, "w") as f:
        json.dump(params, f, indent=1, sort_keys=True)


def load_params(path: str) -> dict:
    with open(path) as f:
        return json.load(f)
