"""Per-kernel-family share of device time from an ncu launch list
(`ncu --metrics gpu__time_duration.sum --csv --log-file X.csv ...`).

  python tools/launch_shares.py gpurun_out/r3g/launches_c2.csv
"""
import collections
import csv
import re
import sys


def family(name):
    m = re.match(r"void bless::k_tc_gemm<(\d+), (\d+), (\d), (\d)>", name)
    if m:
        return f"k_tc_gemm<BN={m.group(1)}, BK={m.group(2)}, halo={m.group(3)}, MH={m.group(4)}>"
    name = re.sub(r"^void ", "", name)
    return re.sub(r"[<(].*", "", name)


def main(path):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
    tot, cnt = collections.Counter(), collections.Counter()
    for r in rows[hi + 1:]:
        if len(r) > vi and r[mi] == "gpu__time_duration.sum":
            f = family(r[ki])
            tot[f] += float(r[vi].replace(",", ""))
            cnt[f] += 1
    T = sum(tot.values())
    print(f"total {T / 1e3:.1f} us of device time over {sum(cnt.values())} launches (ncu: serialised, cold L2)")
    for f, v in tot.most_common():
        print(f"{100 * v / T:5.1f}%  {v / 1e3:9.1f} us  {cnt[f]:5d} launches  {f}")
    tc = sum(v for f, v in tot.items() if f.startswith("k_tc_gemm"))
    halo = sum(v for f, v in tot.items() if "halo=1" in f)
    print(f"tcgen05 conv/GEMM family: {100 * tc / T:.1f}% (halo convs {100 * halo / T:.1f}%)")


if __name__ == "__main__":
    main(sys.argv[1])
