"""Summarise ncu output for profiles/ (run here, on the CPU box).

  python tools/ncu_summary.py launches <launches.csv>          # per-kernel shares of a step
  python tools/ncu_summary.py full <report.ncu-rep> [...]      # key metrics of full captures
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict


def launches(path):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[h]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for r in rows[h + 1:]:
        if len(r) <= vi:
            continue
        name = r[ki]
        for key in ("k_tc_gemm", "k_gemv_tma", "SimtMM", "Pool", "Gemv<", "Eltwise", "k_marker"):
            if key in name:
                name = {"k_tc_gemm": "tc_gemm (tcgen05 GEMM/conv)", "k_gemv_tma": "gemv_tma (TMA weight stream)",
                        "SimtMM": "simt_mm (CUDA-core conv/GEMM)", "Pool": "pool (max/avg/global)",
                        "Gemv<": "gemv_simt", "Eltwise": "eltwise", "k_marker": "marker"}[key]
                break
        else:
            name = name.split("(")[0][:60]
        v = float(r[vi].replace(",", ""))
        if r[ui] == "ms":
            v *= 1e3
        elif r[ui] in ("nsecond", "ns"):
            v /= 1e3
        elif r[ui] in ("usecond", "us"):
            pass
        tot[name] += v
        cnt[name] += 1
    s = sum(tot.values())
    print(f"| kernel family | launches | total us | share |\n|---|---|---|---|")
    for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        print(f"| {k} | {cnt[k]} | {v:.1f} | {100 * v / s:.1f}% |")
    print(f"\nTotal device time {s:.1f} us over {sum(cnt.values())} launches "
          f"(ncu-serialised, cold-cache: compare shares, not absolutes).")


KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__inst_executed_pipe_tensor_subpipe_hmma.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "launch__shared_mem_per_block_dynamic"]


def full(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        print(f"\n**{d.get('Kernel Name', '?')[:90]}** ({path.split('/')[-1]})\n")
        print("| metric | value |\n|---|---|")
        for k in KEYS:
            for hk in hdr:
                if hk.endswith(k) and d.get(hk):
                    print(f"| {k} | {d[hk]} {u.get(hk, '')} |")
                    break


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2])
    else:
        for p in sys.argv[2:]:
            full(p)
