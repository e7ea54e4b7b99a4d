"""Replicas-only multi-GPU path on CPU.

* one process for the box: N CUDA-free contexts (VIRTUAL clock), one box-wide
  trace routed by the native dispatcher (bl_dispatch); every context's
  decisions and completions are bit-exact with the oracle DES run on that
  GPU's slice of the trace;
* one process per GPU (world size 2, gloo): every rank builds the same box
  trace from the gathered per-GPU profiles and runs its own slice, bit-exact
  with the DES; the ranks meet only for the barrier and the max/sum
  reductions bench.py uses -- no data-path collective, no NCCL.
"""
import os
import socket

import numpy as np
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_eurosys_zhangcc0xz0g25_b200 import models, replicas


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _gpu_profile(g, tmpdir):
    """A synthetic B200-scale profile for GPU g's mix (C2/C3/C4 tenant counts)."""
    from synth import profile as sp
    cfg = replicas.plan(g, "C5").config
    rng = np.random.Generator(np.random.PCG64(11 + g))
    spec = models.CONFIGS[cfg]
    tenants = [sp.random_tenant(n, int(round(q * 1e6)), 12 + 4 * j, 148, rng, 4e5, 0.8, 0.1, 1500)
               for j, (n, q) in enumerate(spec)]
    pf = sp.ProfileFile(148, 4, tenants)
    path = os.path.join(tmpdir, f"p{g}.txt")
    sp.save(path, pf)
    return cfg, path, pf


def _box(profs, seed=3, n=6):
    from oracle.sched_ref import Prof
    from synth import trace as tr
    gaps = []
    bursty = []
    for cfg, _, pf in profs:
        prof = Prof(pf)
        gaps.append([prof.T[j] / 0.5 for j in range(prof.ntenants)])
        bursty.append(cfg == "C4")
    return tr.box_trace(gaps, n, seed, bursty)


def _check_gpu(ctx, ids, sub, prof):
    from oracle import des
    from oracle.sched_ref import Params
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi
    recs = ctx.decisions()
    fins = [ctx.poll(r)[1].finish_ns for r in ids]
    ref = des.run_bless(sub, prof, Params(squad_overhead_ns=2000))
    ok = len(recs) == len(ref.decisions) and all(
        capi.decision_to_tuple(r)["picks"] == [tuple(x) for x in d.picks] for r, d in zip(recs, ref.decisions))
    return ok and fins == [ref.finish[i] for i in range(len(sub))]


def test_single_process_box_dispatcher(tmp_path):
    from oracle.sched_ref import Prof
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi
    from synth import trace as tr
    build.build(verbose=False)
    n_gpu = 4
    profs = [_gpu_profile(g, str(tmp_path)) for g in range(n_gpu)]
    box = _box(profs)
    assert [a.arrival_ns for a in box] == sorted(a.arrival_ns for a in box)
    ctxs = []
    for cfg, path, _ in profs:
        c = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, squad_overhead_ns=2000)
        c.load_profile(path)
        ctxs.append(c)
    ents = replicas.dispatch_entries(box, {g: g for g in range(n_gpu)})
    ids = capi.dispatch(ctxs, ents)
    for c in ctxs:
        c.start()
        c.drain(int(30e9))
    for g, (c, (cfg, _, pf)) in enumerate(zip(ctxs, profs)):
        mine = [q for (ci, _, _), q in zip(ents, ids) if ci == g]
        sub = tr.gpu_slice(box, g)
        assert len(mine) == len(sub) > 0
        assert _check_gpu(c, mine, sub, Prof(pf)), g
        c.stop()
        c.close()
    # GPU g's slice does not depend on how many GPUs the box has
    box2 = _box(profs[:2])
    assert tr.gpu_slice(box2, 1) == tr.gpu_slice(box, 1)


def test_dispatcher_rejects_unsorted_and_bad_ctx(tmp_path):
    import pytest
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi
    build.build(verbose=False)
    _, path, _ = _gpu_profile(0, str(tmp_path))
    c = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL)
    c.load_profile(path)
    with pytest.raises(capi.BlessError):
        capi.dispatch([c], [(0, 0, 10), (0, 1, 5)])
    with pytest.raises(capi.BlessError):
        capi.dispatch([c], [(1, 0, 10)])
    c.close()


def _worker(rank, world, port, tmpdir, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle.sched_ref import Prof
        from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi
        from synth import trace as tr
        build.build(verbose=False)
        cfg, path, pf = _gpu_profile(rank, tmpdir)
        # every rank learns every GPU's profile summary, builds the same box trace
        got = replicas.gather((rank, cfg), dist)
        profs = [_gpu_profile(g, tmpdir) for g, _ in sorted(got)]
        box = _box(profs)
        sub = tr.gpu_slice(box, rank)
        ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, squad_overhead_ns=2000)
        ctx.load_profile(path)
        ids = capi.dispatch([ctx], replicas.dispatch_entries(box, {rank: 0}))
        replicas.barrier(dist)
        ctx.start()
        ctx.drain(int(30e9))
        ok = _check_gpu(ctx, ids, sub, Prof(pf))
        fins = [ctx.poll(r)[1].finish_ns for r in ids]
        span = max(fins) - min(a.arrival_ns for a in sub)
        mx = replicas.max_over_ranks(span, dist)
        tot = replicas.sum_over_ranks({"requests": len(ids)}, dist)
        q.put((rank, cfg, ok, span, mx, tot["requests"], len(box)))
        ctx.stop()
        ctx.close()
    finally:
        dist.destroy_process_group()


def test_two_rank_replicas_gloo(tmp_path):
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, str(tmp_path), q)) for r in range(world)]
    for pr in procs:
        pr.start()
    for pr in procs:
        pr.join(180)
        assert pr.exitcode == 0
    res = sorted(q.get(timeout=5) for _ in range(world))
    for rank, cfg, ok, span, mx, tot, nbox in res:
        assert ok, rank                      # each replica bit-exact with the oracle
        assert mx == max(r[3] for r in res)  # max over ranks
        assert tot == nbox                   # whole-job request count = the box trace
    assert [r[1] for r in res] == ["C2", "C3"]   # C5 placement: GPU g hosts C[2 + g mod 3]


def test_plan_c5_mapping():
    got = [replicas.plan(g, "C5").config for g in range(8)]
    assert got == ["C2", "C3", "C4", "C2", "C3", "C4", "C2", "C3"]
    assert all(c in models.CONFIGS for c in got)
    assert replicas.plan(3, "C2").config == "C2"
