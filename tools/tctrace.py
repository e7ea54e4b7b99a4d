"""Phase timeline of the tcgen05 GEMM/conv kernel (debug build with
-DBLESS_TC_TRACE): per-CTA %globaltimer stamps of the last of R back-to-back
launches (programmatic dependent launch on, as in the engine).

  BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE python tools/tctrace.py gemm 384 4096 1024
  BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE python tools/tctrace.py conv 14 14 1024 256 1 1 0

Phases: 0 CTA start, 1 work entry (in range), 2 barriers+TMEM ready, 3 first
claim returned, 4 producer past griddepcontrol.wait, 5 first stage landed
(MMA thread), 6 accumulator ready (epilogue), 7 epilogue stores issued,
8 work done, 9 CTA exit.  Rebuilds the library with the flag (force).
"""
import ctypes as C
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
NAMES = ["start", "entry", "setup", "claim", "pdl_wait", "stage0", "acc_ready", "epi_done", "work_done", "exit",
         "sk_arrived", "sk_reduced"]   # 10/11: split-K units only


def events(L):
    """Per-stage event log of the first CTAs of the last launch: when the
    producer issued each load (after its free-stage wait), when the MMA warp saw
    it land, and when it committed the stage's MMAs."""
    ev = np.zeros((2, 8, 192, 3), dtype=np.uint64)
    cnt = np.zeros((2, 8), dtype=np.int32)
    L.bl_debug_tc_events.argtypes = [C.c_void_p, C.c_void_p]
    L.bl_debug_tc_events(ev.ctypes.data, cnt.ctypes.data)
    ev = ev.astype(np.int64)
    lat = {1: [], 2: []}
    gaps, mwait, pwait = [], [], []
    for cta in range(8):
        nm, npd = cnt[0, cta], cnt[1, cta]
        if nm == 0 or npd == 0:
            continue
        m, pr = ev[0, cta, :nm], ev[1, cta, :npd]
        for kind in (1, 2):
            iss = pr[pr[:, 0] == kind, 2]
            seen = m[m[:, 0] == kind, 2]
            k = min(len(iss), len(seen))
            lat[kind] += list(seen[:k] - iss[:k])
        com = m[m[:, 0] == 9, 1]
        gaps += list(np.diff(com))
        mwait += list(m[m[:, 0] != 9, 2] - m[m[:, 0] != 9, 1])
        pwait += list(pr[:, 2] - pr[:, 1])
        if cta == 0:
            t0 = min(pr[0, 1], m[0, 1])
            print("  CTA 0 event log (us from its first event): P = producer (wait start -> issue), "
                  "M = MMA warp (wait start -> landed), C = commit")
            rows = [(x[1], f"P{'W' if x[0] == 1 else 'H'} {(x[1] - t0) / 1e3:6.2f}->{(x[2] - t0) / 1e3:6.2f}") for x in pr]
            rows += [(x[1], (f"C  {(x[1] - t0) / 1e3:6.2f}" if x[0] == 9 else
                             f"M{'W' if x[0] == 1 else 'H'} {(x[1] - t0) / 1e3:6.2f}->{(x[2] - t0) / 1e3:6.2f}")) for x in m]
            rows.sort()
            line = []
            for _, r in rows:
                line.append(r)
                if len(line) == 5:
                    print("    " + " | ".join(line))
                    line = []
            if line:
                print("    " + " | ".join(line))
    f = lambda a: f"{np.mean(a) / 1e3:.3f}" if len(a) else "-"
    print(f"  (first 8 CTAs) issue -> MMA-warp-sees-landed: weights {f(lat[1])} us, halo {f(lat[2])} us; "
          f"commit-to-commit {f(gaps)} us; MMA warp wait per stage {f(mwait)} us; producer wait per load {f(pwait)} us")


def main():
    assert "BLESS_TC_TRACE" in os.environ.get("BLESS_EXTRA_NVFLAGS", ""), "set BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE"
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi
    from paper_conf_eurosys_zhangcc0xz0g25_b200.models import Builder
    build.build(force=True, verbose=False)
    args = [a for a in sys.argv[1:] if not a.startswith("--act=")]
    act = next((a.split("=")[1] for a in sys.argv[1:] if a.startswith("--act=")), "gelu")
    kind, d = args[0], [int(x) for x in args[1:]]
    ctx = capi.Ctx(0)
    S = ctx.device_info().sm_count
    t = ctx.register_tenant(1.0, "k")
    b = Builder(ctx, t, "k", 1.0, "bf16", seed=7)
    if kind == "gemm":
        b.gemm(b.input((d[0], d[2])), d[1], act=act, bias=True)
    else:
        H, W, Cc, K, k, s, p = d
        b.conv(b.input((1, H, W, Cc)), K, k, s, p, act="relu", bn=True)
    ki = ctx.kernel_info(t, 0)
    L = capi.lib()
    L.bl_debug_tc_trace.argtypes = [C.c_void_p, C.c_int]
    for reps in (1, 20):
        L.bl_debug_tc_trace_clear()
        ns, _ = ctx.profile_kernel(t, 0, S, reps)
        buf = np.zeros((2048, 13), dtype=np.uint64)
        L.bl_debug_tc_trace(buf.ctypes.data, 2048)
        v = buf.astype(np.int64)
        ok = (v[:, 0] > 0) & (v[:, 1] >= v[:, 0]) & (v[:, 9] >= v[:, 1]) & (v[:, 7] > 0)
        w = v[ok]
        t0 = int(v[v[:, 0] > 0, 0].min())
        print(f"{kind} {d} act={act} {ki.family.decode()} tiles={ki.tiles} reps={reps}: event avg {ns / 1e3:.2f} us, "
              f"{ok.sum()} working CTAs")
        if not len(w):
            continue
        print("  phase       min(us)  med(us)  max(us)   (relative to the first CTA start of the last launch)")
        for i, nm in enumerate(NAMES):
            col = w[:, i]
            col = col[col > 0] - t0
            if len(col):
                print(f"  {i} {nm:10s} {col.min() / 1e3:8.2f} {np.median(col) / 1e3:8.2f} {col.max() / 1e3:8.2f}")
        allx = v[v[:, 9] > 0, 9] - t0
        print(f"  last CTA exit (all CTAs) {allx.max() / 1e3:.2f} us")
        rel = w[:, 4] - w[:, 12]
        rel = rel[(w[:, 12] > 0) & (rel > -1e6) & (rel < 1e6)]
        if reps > 1 and len(rel):
            print(f"  griddepcontrol.wait return - predecessor's last CTA exit: min {rel.min() / 1e3:.2f} "
                  f"med {np.median(rel) / 1e3:.2f} max {rel.max() / 1e3:.2f} us")
        if reps > 1:
            events(L)
        if reps == 1:   # wait accounting of that single launch (counters accumulate over launches)
            wb = np.zeros((2048, 4), dtype=np.uint64)
            L.bl_debug_tc_wait.argtypes = [C.c_void_p, C.c_int]
            L.bl_debug_tc_wait(wb.ctypes.data, 2048)
            wb = wb.astype(np.int64)
            on = wb[:, 1] > 0
            if on.any():
                print(f"  MMA warp waiting for operands: {wb[on, 0].mean() / 1e3:.2f} us over "
                      f"{wb[on, 1].mean():.1f} waits; producer waiting for free stages: "
                      f"{wb[on, 2].mean() / 1e3:.2f} us over {wb[on, 3].mean():.1f} waits (per working CTA, "
                      "summed over the profile's launches)")
    ctx.close()


if __name__ == "__main__":
    main()
