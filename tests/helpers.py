"""Small helpers shared by tests (fixture loading only; no method arithmetic)."""
import json
import os

from synth.profile import KernelRow, ProfileFile, TenantRows

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def golden_profile(fx) -> ProfileFile:
    S = fx["S"]
    tenants = []
    for tn in fx["tenants"]:
        rows = []
        if "kernels" in tn:
            for i, k in enumerate(tn["kernels"]):
                rows.append(KernelRow(f"{tn['name']}{i}", k["d"], [k["W"] // min(s, k["d"]) for s in range(1, S + 1)]))
        else:
            for i in range(tn["m"]):
                rows.append(KernelRow(f"{tn['name']}{i}", tn["d"], [tn["t_const"]] * S))
        tenants.append(TenantRows(tn["name"], tn["quota_ppm"], rows, tn.get("slo_ns", 0), tn.get("io_in", 0),
                                  tn.get("io_out", 0)))
    return ProfileFile(S, fx["g"], tenants)
