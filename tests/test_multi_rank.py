"""World-size-2 gloo test of the replicas-only multi-GPU path on CPU
(SURVEY.md §8(e)): each rank runs its own independent C++ scheduler instance
(CUDA-free context, VIRTUAL clock) on its own trace, checks its decisions
bit-exactly against the oracle DES, and the ranks only meet for the barrier and
the max/sum reductions bench.py uses -- no data-path collective."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_eurosys_zhangcc0xz0g25_b200 import replicas


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, tmpdir, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import des
        from oracle.sched_ref import Params, Prof
        from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi
        from synth import profile as sp
        from synth import trace as tr
        build.build(verbose=False)
        p = replicas.plan(rank, world, rank, "C5", ["C2"])
        rng = np.random.Generator(np.random.PCG64(11 + rank))
        tenants = [sp.random_tenant("vgg", 333333, 16, 148, rng, 5e5, 0.8, 0.1, 1500),
                   sp.random_tenant("r50", 666667, 55, 148, rng, 3e5, 0.8, 0.1, 1500)]
        pf = sp.ProfileFile(148, 4, tenants)
        path = os.path.join(tmpdir, f"p{rank}.txt")
        sp.save(path, pf)
        prof = Prof(pf)
        trace = tr.poisson([prof.T[j] / 0.5 for j in range(2)], 12, seed=1 + p.trace_seed_offset)
        ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, squad_overhead_ns=2000)
        ctx.load_profile(path)
        ids = [ctx.submit(a.tenant, a.arrival_ns) for a in trace]
        dist.barrier()
        ctx.start()
        ctx.drain(int(30e9))
        recs = ctx.decisions()
        fins = [ctx.poll(r)[1].finish_ns for r in ids]
        ctx.stop()
        ref = des.run_bless(trace, prof, Params(squad_overhead_ns=2000))
        ok = len(recs) == len(ref.decisions) and all(
            capi.decision_to_tuple(r)["picks"] == [tuple(x) for x in d.picks] for r, d in zip(recs, ref.decisions))
        ok = ok and fins == [ref.finish[i] for i in range(len(trace))]
        span = max(fins) - min(a.arrival_ns for a in trace)
        mx = replicas.max_over_ranks(span, dist)
        tot = replicas.sum_over_ranks({"requests": len(ids)}, dist)
        q.put((rank, p.config, ok, span, mx, tot["requests"]))
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
    for rank, cfg, ok, span, mx, tot in res:
        assert ok, rank                      # each replica bit-exact with the oracle
        assert mx == max(r[3] for r in res)  # max over ranks
        assert tot == 2 * 24                 # whole-job request count
    assert [r[1] for r in res] == ["C2", "C2"]   # C3/C4 not built yet -> C2


def test_plan_c5_mapping():
    got = [replicas.plan(g, 8, g, "C5", ["C2", "C3", "C4"]).config for g in range(8)]
    assert got == ["C2", "C3", "C4", "C2", "C3", "C4", "C2", "C3"]
    assert replicas.plan(3, 4, 3, "C2", ["C2"]).config == "C2"
