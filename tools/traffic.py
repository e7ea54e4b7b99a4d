"""DRAM traffic per kernel (ncu dram__bytes_read/write) mapped onto the
config's (tenant, layer) list, for the bench's roofline `traffic` field.

On the GPU box, under ncu (one process, one GPU):
  ncu --nvtx --nvtx-include "traffic/" --clock-control none --csv \
      --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
      --log-file gpurun_out/traffic_C2.csv \
      python tools/traffic.py launch --config C2 --order gpurun_out/traffic_C2_order.json
Here (CPU):
  python tools/traffic.py reduce --csv gpurun_out/traffic_C2.csv \
      --order gpurun_out/traffic_C2_order.json --out profiles/traffic_C2.json

`launch` launches every kernel of every tenant once, in order, on the full
GPU inside the NVTX range "traffic" (registration-time autotuning and
profiling launches fall outside it).  ncu's default cache control flushes
L2 before each launch, so the bytes are cold-cache: the weights, the input
activations and the output once, plus whatever the kernel re-reads.
"""
import argparse
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def launch(a):
    import torch

    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi, models
    build.build(verbose=False)
    ctx = capi.Ctx(0)
    S = ctx.device_info().sm_count
    ms = models.build_config(ctx, a.config, "fp32" if a.config == "C1" else "bf16")
    order = []
    for m in ms:
        for k in range(len(m.layers)):
            ki = ctx.kernel_info(m.tenant, k)
            order.append({"layer": f"{m.name}[{k}]", "family": ki.family.decode(), "bytes": ki.bytes,
                          "flops": ki.flops})
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_push("traffic")
    for m in ms:
        for k in range(len(m.layers)):
            ctx.run_kernel(m.tenant, k, 0, S)
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_pop()
    json.dump(order, open(a.order, "w"), indent=0)
    print(f"launched {len(order)} kernels")


def reduce(a):
    order = json.load(open(a.order))
    rows = list(csv.reader(open(a.csv)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[h]
    ii, ki, mi, ui, vi = (hdr.index(x) for x in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value"))
    per = {}
    names = {}
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1, "ns": 1, "usecond": 1e3,
             "us": 1e3, "msecond": 1e6, "ms": 1e6}
    for r in rows[h + 1:]:
        if len(r) <= vi:
            continue
        lid = int(r[ii])
        names[lid] = r[ki]
        per.setdefault(lid, {})[r[mi]] = float(r[vi].replace(",", "")) * scale.get(r[ui], 1)
    ids = sorted(per)
    assert len(ids) == len(order), f"{len(ids)} launches in the csv vs {len(order)} kernels"
    out = {}
    for lid, o in zip(ids, order):
        v = per[lid]
        out[o["layer"]] = {"family": o["family"], "kernel": names[lid].split("(")[0],
                           "dram_read": v.get("dram__bytes_read.sum"), "dram_write": v.get("dram__bytes_write.sum"),
                           "ncu_ns": v.get("gpu__time_duration.sum"), "algorithmic_bytes": o["bytes"],
                           "algorithmic_flops": o["flops"]}
    json.dump({"source": os.path.basename(a.csv), "note": "ncu per-launch dram bytes, cold L2 (cache-control all), "
               "each kernel alone on all SMs", "layers": out}, open(a.out, "w"), indent=1)
    tot_r = sum(x["dram_read"] + x["dram_write"] for x in out.values())
    tot_a = sum(x["algorithmic_bytes"] for x in out.values())
    print(f"{len(out)} kernels: dram {tot_r / 1e6:.1f} MB vs algorithmic {tot_a / 1e6:.1f} MB")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("mode", choices=["launch", "reduce"])
    ap.add_argument("--config", default="C2")
    ap.add_argument("--order", required=True)
    ap.add_argument("--csv")
    ap.add_argument("--out")
    a = ap.parse_args()
    launch(a) if a.mode == "launch" else reduce(a)


if __name__ == "__main__":
    main()
